# Round measurement: tests, smoke, bench (default), per-op profile, ncu launch list
# (dram bytes + time) of the bench command, ncu --set full of the top kernels.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/gputests.log 2>&1; echo tests=$?
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; echo bench=$?
timeout 300 python tools/opprofile.py > gpurun_out/opprofile.log 2>&1; echo opp=$?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv python bench.py --profile-only > gpurun_out/ncu_launches.log 2>&1; echo ncu1=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -s 8 -c 5 -o gpurun_out/full_ssb41 python tools/opprofile.py --queries ssb4.1 --launch 1 > gpurun_out/ncu_full.log 2>&1; echo ncu2=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:agg_ws -s 2 -c 1 -o gpurun_out/full_agg11 python tools/opprofile.py --queries ssb1.1 --launch 1 >> gpurun_out/ncu_full.log 2>&1; echo ncu3=$?
