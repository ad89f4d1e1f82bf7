# ncu --set full of Q3.1's and Q4.1's operators (dense probe, at-TIDs probes, fetch,
# aggregate) and Q1.1's aggregate at SF20, for the round-2 kernel analysis
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"ws_kernel|agg_ws|fetch_kernel|join_index_build" -c 8 -o gpurun_out/r2_full_ssb31 python tools/opprofile.py --queries ssb3.1 --launch 1 > gpurun_out/r2_ncu31.log 2>&1; echo a=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"ws_kernel|agg_ws|fetch_kernel" -c 8 -o gpurun_out/r2_full_ssb41 python tools/opprofile.py --queries ssb4.1 --launch 1 > gpurun_out/r2_ncu41.log 2>&1; echo b=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"agg_ws" -c 2 -o gpurun_out/r2_full_ssb11 python tools/opprofile.py --queries ssb1.1 --launch 1 > gpurun_out/r2_ncu11.log 2>&1; echo c=$?
for f in gpurun_out/r2_full_*.ncu-rep; do python tools/ncu_summary2.py $f > ${f%.ncu-rep}.txt 2>&1; done
