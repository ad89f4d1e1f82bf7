# Per-rank step of W-GPU runs emulated on one B200 (rank 0's data; no exchange):
# weak scaling (SF 20*W, 120 M rows per rank) and strong scaling (SF100 split W ways)
set -x
mkdir -p gpurun_out
for W in 2 4 8; do
  timeout 900 python bench.py --no-e2e --no-cpu-baseline --emulate-world $W >> gpurun_out/se_weak.jsonl 2>> gpurun_out/se.err; echo weak$W=$?
done
for W in 2 4 8; do
  timeout 900 python bench.py --no-e2e --no-cpu-baseline --sf-total 100 --emulate-world $W >> gpurun_out/se_strong.jsonl 2>> gpurun_out/se.err; echo strong$W=$?
done
