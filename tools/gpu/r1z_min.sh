timeout 900 python -m pytest tests/test_gpu_tpch.py tests/test_gpu_ops.py -x -q > gpurun_out/r1z_min_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r1z_min_tests.log
tail -n 25 gpurun_out/r1z_min_tests.log
