# ncu --set full of the dense probe kernel (microbench, 120M keys, 73 KB bitmap, 20 % pass, payload emitted)
set -x
timeout 600 python -m pytest tests -m gpu -x -q -k "probe or ssb" > gpurun_out/gputests.log 2>&1; echo tests=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dense_probe -s 3 -c 1 -o gpurun_out/dp_full python tools/microbench.py "bitmap73KB pass 0.20 emit=True" > gpurun_out/ncu_dp.log 2>&1; echo ncu=$?
