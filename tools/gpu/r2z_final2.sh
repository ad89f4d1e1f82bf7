# Final validation at HEAD: GPU suite, smoke, default bench x2, SF100 bench, TPC-H SF30, M1
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/g_gputests.log 2>&1; echo tests=$?
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g_smoke.log 2>&1; echo smoke=$?
for i in 1 2; do timeout 900 python bench.py >> gpurun_out/g_bench_sf20.jsonl 2>> gpurun_out/g_bench.err; echo bench=$?; done
timeout 1200 python bench.py --sf 100 --no-e2e --no-cpu-baseline >> gpurun_out/g_bench_sf100.jsonl 2>> gpurun_out/g_bench.err; echo b100=$?
timeout 900 python tools/tpch_bench.py > gpurun_out/g_tpch_sf30.jsonl 2> gpurun_out/g_tpch.err; echo tpch=$?
timeout 600 python tools/driver_profile.py --queries tpch2 --cold > gpurun_out/g_dp.txt 2>&1; echo dp=$?
