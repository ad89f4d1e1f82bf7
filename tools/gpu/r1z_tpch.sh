set -x
timeout 900 python -m pytest tests/test_gpu_tpch.py -x -q > gpurun_out/r1z_tpch_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r1z_tpch_tests.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q -k tpch > gpurun_out/r1z_tpch_full.log 2>&1; echo "rc=$?" >> gpurun_out/r1z_tpch_full.log
timeout 900 python tools/tpch_bench.py --sf 30 --ops > gpurun_out/r1z_tpch_bench.jsonl 2> gpurun_out/r1z_tpch_bench.err
tail -n 15 gpurun_out/r1z_tpch_tests.log gpurun_out/r1z_tpch_full.log
cut -c1-400 gpurun_out/r1z_tpch_bench.jsonl
