python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/tpch_q1_launch.py --sf 30 --time > gpurun_out/q1_time.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:agg_dense -c 1 -o gpurun_out/q1_dense python tools/tpch_q1_launch.py --sf 10 --launch 1 > gpurun_out/q1_ncu.log 2>&1; echo rc=$?
