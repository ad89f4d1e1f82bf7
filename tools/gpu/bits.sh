set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; echo tests=$?
timeout 300 python tools/opprofile.py > gpurun_out/opprofile.log 2>&1; echo opp=$?
DDQ_ROW_BITMAPS=0 timeout 300 python tools/opprofile.py > gpurun_out/opprofile_nobits.log 2>&1; echo opp=$?
timeout 600 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench.log 2>&1; echo bench=$?
timeout 600 python bench.py --no-e2e --no-cpu-baseline --streams 4 > gpurun_out/bench_s4.log 2>&1; echo bench=$?
