python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python tools/opprofile.py --sf 100 --queries ssb3.1,ssb4.1,ssb4.2 > gpurun_out/opprofile_sf100b.txt 2>&1
timeout 900 python bench.py --no-cpu-baseline --no-e2e --sf 100 > gpurun_out/bench_sf100b.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_sf20b.log 2>&1
timeout 900 python -m pytest tests/test_gpu_ssb.py tests/test_gpu_coarse.py tests/test_gpu_sparse.py -q -x 2>&1 | tail -2 > gpurun_out/t53.log
