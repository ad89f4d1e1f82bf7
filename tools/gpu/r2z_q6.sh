set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -k "tpch or sparse" > gpurun_out/q6_tests.log 2>&1; echo tests=$?
timeout 900 python tools/tpch_bench.py --ops > gpurun_out/q6_tpch.jsonl 2> gpurun_out/q6_tpch.err; echo tp=$?
