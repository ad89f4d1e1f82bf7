for P in "" "0,-1,-1" "-1,0,0" "" "0,-1,-1" "-1,-1,0"; do
  DDQ_LANE_PRIO=$P timeout 300 python bench.py --no-e2e --no-cpu-baseline --streams 4 --steps 50 > /tmp/o.json 2>/dev/null
  echo "[$P] $(tail -1 /tmp/o.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'])")" >> gpurun_out/prio.txt
done
