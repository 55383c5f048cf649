# PSIM_TIMING timelines (step 900, G = 8 slice) of timing-build variants tools/gpu/ab/<v>.so
mkdir -p gpurun_out
for v in $1; do
  PSIM_LIB=tools/gpu/ab/$v.so PSIM_DEBUG_TIMING=900 PSIM_DEBUG_TIMING_OUT=gpurun_out/timing_e8_$v.txt timeout 600 python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu --emulate-rank 0/8 2>&1 | tail -1 | cut -c1-50
done
