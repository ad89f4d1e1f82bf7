set -x
timeout 300 python tools/opprofile.py > gpurun_out/opprofile.log 2>&1; echo opp=$?
timeout 300 python tools/opprofile.py --queries ssb3.1,ssb4.1 > gpurun_out/opprofile_b.log 2>&1; echo opp=$?
timeout 600 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo bench=$?
