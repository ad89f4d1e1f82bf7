set -x
mkdir -p gpurun_out
for W in 2 4 8; do
  timeout 900 python bench.py --no-e2e --no-cpu-baseline --sf-total 100 --emulate-world $W >> gpurun_out/st_strong.jsonl 2>> gpurun_out/st.err; echo strong$W=$?
done
timeout 900 python tools/opprofile.py --sf 12.5 --world 8 > gpurun_out/st_w8_opprofile.txt 2>&1; echo opp=$?
timeout 900 python tools/timeline.py --sf 100 --streams 1 --out gpurun_out/st_tl_sf100.json > /dev/null 2>&1; echo tl=$?
