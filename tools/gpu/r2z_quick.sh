# quick A/B: build/probe/query parity subset, 2 bench runs (hot only), timeline
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "ssb or tpch or ops or sparse or coarse" > gpurun_out/q_tests.log 2>&1; echo tests=$?
for i in 1 2; do timeout 300 python bench.py --no-e2e --no-cpu-baseline --steps 50 > gpurun_out/q_bench$i.log 2>&1; echo bench=$?; done
timeout 300 python tools/timeline.py --streams 1 --out gpurun_out/q_tl1.json > gpurun_out/q_tl.log 2>&1
timeout 300 python tools/timeline.py --streams 4 --out gpurun_out/q_tl4.json >> gpurun_out/q_tl.log 2>&1
