set -x
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_ops.py -x -q > gpurun_out/b_ops.log 2>&1; echo ops=$?
timeout 300 python tools/timeline.py --streams 1 --out gpurun_out/b_tl1.json > /dev/null 2>&1
timeout 900 python tools/timeline.py --sf 100 --streams 1 --out gpurun_out/b_tl100.json > /dev/null 2>&1
