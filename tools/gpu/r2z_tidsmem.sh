set -x
for T in "" 160000 100000; do
  echo "== T=$T" >> gpurun_out/ts_opp.txt
  DDQ_WS_TID_SMEM_MAX=$T timeout 900 python tools/opprofile.py --world 4 --queries ssb4.1,ssb2.1,ssb4.3 >> gpurun_out/ts_opp.txt 2>&1
  DDQ_WS_TID_SMEM_MAX=$T timeout 900 python bench.py --no-e2e --no-cpu-baseline --emulate-world 4 >> gpurun_out/ts_bench.jsonl 2>/dev/null
  DDQ_WS_TID_SMEM_MAX=$T timeout 900 python bench.py --no-e2e --no-cpu-baseline >> gpurun_out/ts_bench.jsonl 2>/dev/null
done
