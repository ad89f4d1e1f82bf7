# M5 at spec re-run at the final HEAD (dictionary transfer code, masked probes over L2)
set -x
mkdir -p gpurun_out
timeout 2400 python tools/config5.py > gpurun_out/r2z_config5_sf20.jsonl 2> gpurun_out/r2z_config5.err; echo m5=$?
