python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for S in 1 2 3 4 5 6 8 13; do
  timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 50 --streams $S > /tmp/o.json 2>/dev/null
  echo "streams=$S $(tail -1 /tmp/o.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'])")"
done
