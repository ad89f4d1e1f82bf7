set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r1z_gputests.log 2>&1; echo "tests rc=$?" >> gpurun_out/r1z_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1z_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r1z_smoke.log
for i in 1 2; do timeout 600 python bench.py >> gpurun_out/r1z_bench.jsonl 2>> gpurun_out/r1z_bench.err; done
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r1z_launches.csv python bench.py --profile-only > gpurun_out/r1z_ncu_bench.log 2>&1
tail -3 gpurun_out/r1z_gputests.log gpurun_out/r1z_smoke.log
cut -c1-300 gpurun_out/r1z_bench.jsonl
