set -x
./tools/cuda/gather_probe > gpurun_out/gather_probe.log 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --csv --log-file gpurun_out/gather_ncu.csv ./tools/cuda/gather_probe > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; echo tests=$?
timeout 300 python tools/opprofile.py > gpurun_out/opprofile.log 2>&1; echo opp=$?
timeout 600 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo bench=$?
