# A/B: O37 fused tails for a subset of the SSB queries in the 4-stream bench step
for S in "" "ssb2.2,ssb2.3,ssb3.3,ssb3.4" "ssb2.1,ssb2.2,ssb2.3,ssb3.2,ssb3.3,ssb3.4,ssb4.3" "ssb2.3,ssb3.3,ssb3.4" ""; do
  for r in 1 2; do
  DDQ_FUSE_TAIL=$S timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 50 > /tmp/o.json 2>/dev/null
  echo "[$S] $(tail -1 /tmp/o.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['config']['serial_ms_per_step'])")" >> gpurun_out/ft.txt
  done
done
