# compute-sanitizer over the hot-path kernels: memcheck on the small and
# medium runs, racecheck / synccheck on the small run (shared-memory hazards, barrier misuse)
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck synccheck; do
  timeout 900 $CS --tool $tool --print-limit 20 python tools/gpu/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?"; tail -3 gpurun_out/sanitize_$tool.log
done
timeout 1200 $CS --tool racecheck --racecheck-report hazard --print-limit 20 python tools/gpu/sanitize_run.py small > gpurun_out/sanitize_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -3 gpurun_out/sanitize_racecheck.log
timeout 900 $CS --tool initcheck --print-limit 20 python tools/gpu/sanitize_run.py small > gpurun_out/sanitize_initcheck.log 2>&1; echo "initcheck rc=$?"; tail -3 gpurun_out/sanitize_initcheck.log
