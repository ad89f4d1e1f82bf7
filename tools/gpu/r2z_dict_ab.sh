# A/B: dictionary transfer code on the cold paths (SSB e2e, TPC-H SF30 cold)
set -x
mkdir -p gpurun_out
python tools/h2d_probe.py > gpurun_out/d_h2d.txt 2>&1
for D in 1 0 1 0; do
  DDQ_TRANSFER_DICT=$D timeout 600 python bench.py --no-cpu-baseline --steps 3 >> gpurun_out/d_bench_$D.jsonl 2>/dev/null; echo b$D=$?
done
for D in 1 0; do DDQ_TRANSFER_DICT=$D timeout 900 python tools/tpch_bench.py > gpurun_out/d_tpch_$D.jsonl 2>/dev/null; echo t$D=$?; done
