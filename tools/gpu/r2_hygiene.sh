# compute-sanitizer over every kernel family, M1, and the bench's new cpu_baseline
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  timeout 1500 $CS --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_run.py > gpurun_out/r2_sanitize_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/r2_sanitize_rc.txt
done
timeout 600 python tools/m1.py --out gpurun_out/r2_m1.json > gpurun_out/r2_m1.log 2>&1; echo m1=$?
