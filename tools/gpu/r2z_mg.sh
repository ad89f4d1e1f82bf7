# A/B: bitmap-masked probes of join indexes in L2 (DDQ_MASKED_GLOBAL) at SF80 / SF160 dims and SF100
set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -k "ssb or coarse or sparse or fullsize or dist" > gpurun_out/mg_tests.log 2>&1; echo tests=$?
for MG in 1 0; do
for W in 4 8; do
  DDQ_MASKED_GLOBAL=$MG timeout 900 python bench.py --no-e2e --no-cpu-baseline --emulate-world $W >> gpurun_out/mg_$MG.jsonl 2>> gpurun_out/mg.err; echo w$W=$?
done
DDQ_MASKED_GLOBAL=$MG timeout 1200 python bench.py --no-e2e --no-cpu-baseline --sf 100 >> gpurun_out/mg_$MG.jsonl 2>> gpurun_out/mg.err; echo sf100=$?
done
DDQ_MASKED_GLOBAL=1 timeout 900 python tools/opprofile.py --world 4 > gpurun_out/mg_w4_opprofile.txt 2>&1
