# racecheck with every hazard printed, reduced on the box to the unique (kernel:line) pairs
mkdir -p gpurun_out
timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 10000000 \
  python tools/gpu/sanitize_run.py small 2>&1 | grep -A2 "Potential" | grep -o "Write Thread.*\|Read Thread.*" \
  | sed 's/Thread ([0-9,]*)//; s/+0x[0-9a-f]*//; s/(CUtensor[^)]*)//' | paste - - | sort | uniq -c > gpurun_out/racecheck_pairs.txt
echo "racecheck done"; cat gpurun_out/racecheck_pairs.txt | head -20
