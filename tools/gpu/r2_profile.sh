# Round-2 profile refresh at SF20: the ncu launch list of the bench command (per-class
# DRAM bytes and device time), the event-timed per-operator profile with the S8(d)
# algorithmic bytes, and ncu --set full of Q3.1's / Q4.1's / Q1.1's operators.
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_launches_bench.csv python bench.py --profile-only > gpurun_out/r2_ncu_launches.log 2>&1; echo l=$?
timeout 600 python tools/opprofile.py --json gpurun_out/r2_opprofile_sf20.json > gpurun_out/r2_opprofile_sf20.txt 2>&1; echo o=$?
bash tools/gpu/r2_ncu.sh
