# dense probe kernel: parity tests + microbench old vs new + opprofile
set -x
./tools/cuda/atomic_rate > gpurun_out/atomic_rate.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "probe or ssb" > gpurun_out/gputests.log 2>&1; echo tests=$?
DDQ_DENSE_PROBE=0 timeout 300 python tools/microbench.py probe > gpurun_out/mb_old.log 2>&1
timeout 300 python tools/microbench.py probe > gpurun_out/mb_new.log 2>&1
timeout 300 python tools/opprofile.py > gpurun_out/opprofile.log 2>&1; echo opp=$?
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo bench=$?
