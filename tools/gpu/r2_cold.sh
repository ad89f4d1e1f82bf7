set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests/test_gpu_tpch.py tests/test_gpu_transfer.py tests/test_gpu_driver.py -q -x > gpurun_out/r2_cold_tests.log 2>&1; echo t=$?
timeout 900 python tools/tpch_bench.py > gpurun_out/r2_tpch_sf30.jsonl 2> gpurun_out/r2_tpch.err; echo tpch=$?
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r2_bench_prefetch.log 2>&1; echo b1=$?
timeout 900 python bench.py --no-cpu-baseline --no-prefetch > gpurun_out/r2_bench_noprefetch.log 2>&1; echo b2=$?
