# M5 at spec (SF20, 104 queries, U in {1,8,16,32}, five arms) and the App. E / Fig. 24
# cache sweep (SF10, LFU vs LRU, cache 0..100 % of the working set, DDC, 8 users)
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests/test_gpu_driver.py -q > gpurun_out/r2_driver_tests.log 2>&1; echo drv=$?
nproc > gpurun_out/r2_m5_host.txt
timeout 2400 python tools/config5.py > gpurun_out/r2_config5_sf20.jsonl 2> gpurun_out/r2_config5.err; echo m5=$?
for frac in 0 0.25 0.5 0.75 1.0; do
  for pol in lfu lru; do
    timeout 600 python tools/config5.py --sf 10 --arms ddc --users 8 --cache-frac $frac --policy $pol >> gpurun_out/r2_fig24_sf10.jsonl 2>> gpurun_out/r2_fig24.err
  done
done
echo fig24=$?
