python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:agg_ws -c 2 -o gpurun_out/agg11_bits python tools/opprofile.py --queries ssb1.1 --launch 1 > gpurun_out/agg11.log 2>&1; echo rc=$?
DDQ_ROW_BITMAPS=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:agg_ws -c 2 -o gpurun_out/agg11_tids python tools/opprofile.py --queries ssb1.1 --launch 1 >> gpurun_out/agg11.log 2>&1; echo rc=$?
