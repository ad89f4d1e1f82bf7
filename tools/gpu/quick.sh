# quick A/B: per-operator profile of the named queries + the default bench (no e2e/cpu)
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/opprofile.py --queries ${Q:-ssb3.1,ssb4.2,ssb4.1} > gpurun_out/quick_opprofile.txt 2>&1
for r in 1 2; do
timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 50 > /tmp/o.json 2>/dev/null
echo "bench $(tail -1 /tmp/o.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['config']['serial_ms_per_step'])")" >> gpurun_out/quick_opprofile.txt
done
