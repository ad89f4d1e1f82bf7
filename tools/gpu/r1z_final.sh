set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r1z_final_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r1z_final_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1z_final_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r1z_final_smoke.log
timeout 600 python bench.py > gpurun_out/r1z_final_bench.jsonl 2> gpurun_out/r1z_final_bench.err
timeout 600 python bench.py --impl reference > gpurun_out/r1z_final_ref.jsonl 2> gpurun_out/r1z_final_ref.err
tail -n 3 gpurun_out/r1z_final_tests.log gpurun_out/r1z_final_smoke.log
cut -c1-250 gpurun_out/r1z_final_bench.jsonl gpurun_out/r1z_final_ref.jsonl
