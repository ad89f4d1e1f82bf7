python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for C in unset 100 72 58 unset 100; do
  if [ "$C" = unset ]; then unset DDQ_CARVEOUT; else export DDQ_CARVEOUT=$C; fi
  timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 50 > /tmp/o.json 2>/dev/null
  echo "carveout=$C $(tail -1 /tmp/o.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['config']['serial_ms_per_step'])")"
done
