set -x
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_ops.py -x -q > gpurun_out/i_ops.log 2>&1; echo ops=$?
timeout 900 python -m pytest tests -m gpu -x -q -k "tpch or ssb or sparse or coarse" > gpurun_out/i_tests.log 2>&1; echo tests=$?
for B in 1 0; do
  DDQ_BUILD_ILP=$B timeout 900 python tools/tpch_bench.py --ops > gpurun_out/i_tpch_$B.jsonl 2> gpurun_out/i_tpch_$B.err; echo tp$B=$?
  DDQ_BUILD_ILP=$B timeout 300 python tools/timeline.py --streams 1 --out gpurun_out/i_tl_$B.json > /dev/null 2>&1
  DDQ_BUILD_ILP=$B timeout 900 python bench.py --no-e2e --no-cpu-baseline --sf 100 >> gpurun_out/i_bench.jsonl 2>/dev/null; echo b$B=$?
  DDQ_BUILD_ILP=$B timeout 900 python bench.py --no-e2e --no-cpu-baseline >> gpurun_out/i_bench.jsonl 2>/dev/null; echo b$B=$?
done
