# Final validation at HEAD (round-2 end): GPU suite, smoke, default bench x2, SF100 bench
set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/z_gputests.log 2>&1; echo tests=$?
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/z_smoke.log 2>&1; echo smoke=$?
for i in 1 2; do timeout 900 python bench.py >> gpurun_out/z_bench_sf20.jsonl 2>> gpurun_out/z_bench.err; echo bench=$?; done
timeout 1200 python bench.py --sf 100 --no-cpu-baseline >> gpurun_out/z_bench_sf100.jsonl 2>> gpurun_out/z_bench.err; echo b100=$?
