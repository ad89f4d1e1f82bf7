# Round-2 baseline: bench (default), per-op profile, ncu launch list of the bench command
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r2_bench.log 2>&1; echo bench=$?
timeout 300 python tools/opprofile.py > gpurun_out/r2_opprofile.log 2>&1; echo opp=$?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_launches_bench.csv python bench.py --profile-only > gpurun_out/r2_ncu_launches.log 2>&1; echo ncu1=$?
