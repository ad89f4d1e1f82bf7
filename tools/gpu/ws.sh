# warp-autonomous filter kernels: parity + microbench + per-op profile + bench
set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; echo tests=$?
timeout 300 python tools/microbench.py probe > gpurun_out/mb_new.log 2>&1
timeout 300 python tools/opprofile.py > gpurun_out/opprofile.log 2>&1; echo opp=$?
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo bench=$?
