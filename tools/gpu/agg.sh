set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; echo tests=$?
timeout 300 python tools/opprofile.py > gpurun_out/opprofile.log 2>&1; echo opp=$?
DDQ_AGG_WS=0 timeout 300 python tools/opprofile.py > gpurun_out/opprofile_oldagg.log 2>&1; echo opp=$?
timeout 600 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo bench=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:agg_ws -s 2 -c 1 -o gpurun_out/agg11 python tools/opprofile.py --queries ssb1.1 --launch 1 > gpurun_out/ncu_agg.log 2>&1; echo ncu=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:agg_ws -s 2 -c 1 -o gpurun_out/agg31 python tools/opprofile.py --queries ssb3.1 --launch 1 >> gpurun_out/ncu_agg.log 2>&1; echo ncu=$?
