python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:ws_kernel<\(int\)0, \(int\)2, \(bool\)1' -c 1 -o gpurun_out/k2pay python tools/opprofile.py --queries ssb3.1 --launch 1 > gpurun_out/k2pay.log 2>&1; echo rc=$?
