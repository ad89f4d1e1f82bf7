timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r1z_ks_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r1z_ks_tests.log
timeout 900 python tools/tpch_bench.py --sf 30 --ops > gpurun_out/r1z_ks_tpch.jsonl 2> gpurun_out/r1z_ks_tpch.err
timeout 600 python bench.py > gpurun_out/r1z_ks_bench.jsonl 2> gpurun_out/r1z_ks_bench.err
tail -n 2 gpurun_out/r1z_ks_tests.log
grep '"hot"' gpurun_out/r1z_ks_tpch.jsonl | cut -c1-140
grep tpch4 gpurun_out/r1z_ks_tpch.err
cut -c1-160 gpurun_out/r1z_ks_bench.jsonl
