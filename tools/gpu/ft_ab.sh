for S in "" "ssb2.2,ssb2.3,ssb3.3,ssb3.4" "ssb2.3,ssb3.3,ssb3.4" "ssb2.2,ssb2.3,ssb3.3,ssb3.4,ssb4.3" "" ; do
  for r in 1 2; do
  FT_SET=$S timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 50 > /tmp/o.json 2>/dev/null
  echo "$S $(tail -1 /tmp/o.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['config']['serial_ms_per_step'])")"
  done
done
