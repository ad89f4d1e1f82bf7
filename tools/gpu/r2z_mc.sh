set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -k "coarse or fullsize or ssb" > gpurun_out/mc_tests.log 2>&1; echo tests=$?
for M in 1 0 1 0; do
  DDQ_MASKED_COARSE=$M timeout 900 python bench.py --no-e2e --no-cpu-baseline --sf 100 >> gpurun_out/mc_$M.jsonl 2>/dev/null; echo b$M=$?
done
DDQ_MASKED_COARSE=1 timeout 900 python bench.py --no-e2e --no-cpu-baseline --emulate-world 8 >> gpurun_out/mc_1.jsonl 2>/dev/null
DDQ_MASKED_COARSE=0 timeout 900 python bench.py --no-e2e --no-cpu-baseline --emulate-world 8 >> gpurun_out/mc_0.jsonl 2>/dev/null
