set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -k "tpch or sparse or ssb or ops or fullsize" > gpurun_out/sb_tests.log 2>&1; echo tests=$?
DDQ_ROW_BITMAPS=1 timeout 900 python tools/tpch_bench.py --ops > gpurun_out/sb_tpch.jsonl 2> gpurun_out/sb_tpch.err; echo tp=$?
timeout 600 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/sb_bench.jsonl 2>/dev/null; echo b=$?
