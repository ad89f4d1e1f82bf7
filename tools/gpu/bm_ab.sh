for V in 1 2 1 2; do
  DDQ_ROW_BITMAPS=$V timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 50 > /tmp/o.json 2>/dev/null
  echo "bm=$V $(tail -1 /tmp/o.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['config']['serial_ms_per_step'])")"
done
DDQ_ROW_BITMAPS=2 timeout 300 python tools/opprofile.py --queries ssb3.1,ssb4.2,ssb4.1 > gpurun_out/bm2_opprofile.txt 2>&1
DDQ_ROW_BITMAPS=1 timeout 300 python tools/opprofile.py --queries ssb3.1,ssb4.2,ssb4.1 > gpurun_out/bm1_opprofile.txt 2>&1
