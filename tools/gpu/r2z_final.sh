# Final round-2 measurement at HEAD: GPU suite, smoke, default bench x2, SF100 bench,
# TPC-H SF30 hot/cold, M1, the oracle reference arm
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/f_gpu.txt
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/f_gputests.log 2>&1; echo tests=$?
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f_smoke.log 2>&1; echo smoke=$?
for i in 1 2; do timeout 900 python bench.py >> gpurun_out/f_bench_sf20.jsonl 2>> gpurun_out/f_bench.err; echo bench=$?; done
timeout 1200 python bench.py --sf 100 --no-e2e --no-cpu-baseline >> gpurun_out/f_bench_sf100.jsonl 2>> gpurun_out/f_bench.err; echo b100=$?
timeout 900 python tools/tpch_bench.py > gpurun_out/f_tpch_sf30.jsonl 2> gpurun_out/f_tpch.err; echo tpch=$?
timeout 600 python tools/m1.py --out gpurun_out/f_m1.json > gpurun_out/f_m1.log 2>&1; echo m1=$?
timeout 600 python bench.py --impl reference > gpurun_out/f_bench_reference.jsonl 2>> gpurun_out/f_bench.err; echo ref=$?
