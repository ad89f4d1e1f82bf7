set -x
mkdir -p gpurun_out
timeout 600 python tools/timeline.py --streams 4 --out gpurun_out/tl4.json > gpurun_out/tl.log 2>&1; echo tl4=$?
timeout 600 python tools/timeline.py --streams 1 --out gpurun_out/tl1.json >> gpurun_out/tl.log 2>&1; echo tl1=$?
