set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_driver.py tests/test_gpu_ssb.py -q -k "placement or driver or admission or chopping or fig" > gpurun_out/r2_m5b_tests.log 2>&1; echo t=$?
timeout 2400 python tools/config5.py --arms chopping,gpu_only,ddc > gpurun_out/r2_config5_sf20_oldest.jsonl 2> gpurun_out/r2_config5b.err; echo m5=$?
