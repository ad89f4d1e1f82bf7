# Session re-entry baseline at HEAD: GPU suite, smoke, default bench
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt
free -g > gpurun_out/free.txt; nproc >> gpurun_out/free.txt
timeout 1500 python -m pytest tests -m gpu -q --durations=25 > gpurun_out/gputests.log 2>&1; echo tests=$?
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; echo bench=$?
