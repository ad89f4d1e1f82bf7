set -x
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_ops.py -x -q > gpurun_out/b_ops.log 2>&1; echo ops=$?
timeout 900 python -m pytest tests -m gpu -x -q -k "ssb or tpch or sparse or coarse" > gpurun_out/b_tests.log 2>&1; echo tests=$?
for i in 1 2; do timeout 300 python bench.py --no-e2e --no-cpu-baseline --steps 50 >> gpurun_out/b_bench.jsonl 2>/dev/null; done
timeout 900 python bench.py --no-e2e --no-cpu-baseline --sf-total 100 --emulate-world 8 >> gpurun_out/b_bench.jsonl 2>/dev/null
timeout 300 python tools/timeline.py --streams 1 --out gpurun_out/b_tl1.json > /dev/null 2>&1
