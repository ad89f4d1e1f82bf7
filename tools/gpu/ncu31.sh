set -x
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -s 8 -c 4 -o gpurun_out/ws31b python tools/opprofile.py --queries ssb3.1 --launch 1 > gpurun_out/ncu_ws31b.log 2>&1; echo ncu=$?
