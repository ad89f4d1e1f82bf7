# Round-2 (final session) profile refresh at SF20: ncu launch list of the bench command
# (per-class DRAM bytes + device time), event-timed per-operator profile with the S8(d)
# bytes, CUPTI timelines (1 and 4 streams), ncu --set full of Q3.1's / Q1.1's graph-
# launched kernels (the capture skips data-load kernels by name; eager + graph halves)
set -x
mkdir -p gpurun_out
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2z_launches_bench.csv python bench.py --profile-only > gpurun_out/r2z_ncu_launches.log 2>&1; echo l=$?
timeout 600 python tools/opprofile.py --json gpurun_out/r2z_opprofile_sf20.json > gpurun_out/r2z_opprofile_sf20.txt 2>&1; echo o=$?
timeout 300 python tools/timeline.py --streams 1 --out gpurun_out/r2z_tl1.json > gpurun_out/r2z_tl.log 2>&1
timeout 300 python tools/timeline.py --streams 4 --out gpurun_out/r2z_tl4.json >> gpurun_out/r2z_tl.log 2>&1
for Q in ssb3.1 ssb1.1; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"ws_kernel|agg_ws|fetch_kernel|join_index_build|multi_fill|groupby_compact" -c 24 -o /tmp/r2z_full_$Q python tools/opprofile.py --queries $Q --launch 1 > gpurun_out/r2z_ncu_$Q.log 2>&1; echo $Q=$?
python tools/ncu_summary2.py /tmp/r2z_full_$Q.ncu-rep > gpurun_out/r2z_full_$Q.txt 2>&1
done
