# ncu --set full of every kernel of one eager run + one graph launch of SSB Q4.1 / Q3.1
# at SF20 (the graph-launched half is what bench.py runs); reports summarised on the box
set -x
mkdir -p gpurun_out
for Q in ssb4.1 ssb3.1; do
timeout 900 ncu --set full --clock-control none --import-source on -c 40 -o /tmp/r2z_full_$Q python tools/opprofile.py --queries $Q --launch 1 > gpurun_out/r2z_ncu_$Q.log 2>&1; echo $Q=$?
python tools/ncu_summary2.py /tmp/r2z_full_$Q.ncu-rep > gpurun_out/r2z_full_$Q.txt 2>&1
ncu -i /tmp/r2z_full_$Q.ncu-rep --page source --csv --print-source sass -k regex:agg_ws > gpurun_out/r2z_src_agg_$Q.csv 2>/dev/null
done
ls -la /tmp/*.ncu-rep
