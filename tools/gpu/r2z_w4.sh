set -x
mkdir -p gpurun_out
for W in 2 4 8; do timeout 900 python tools/opprofile.py --world $W > gpurun_out/w${W}_opprofile.txt 2>&1; echo w$W=$?; done
