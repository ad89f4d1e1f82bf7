set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; echo tests=$?
timeout 300 python tools/microbench.py probe > gpurun_out/mb_new.log 2>&1
timeout 300 python tools/opprofile.py > gpurun_out/opprofile.log 2>&1; echo opp=$?
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo bench=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -s 8 -c 4 -o gpurun_out/ws31 python tools/opprofile.py --queries ssb3.1 --launch 1 > gpurun_out/ncu_ws31.log 2>&1; echo ncu=$?
