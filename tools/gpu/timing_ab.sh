# PSIM_TIMING timelines (step 900, G = 8 slice and G = 1) of the in-tree timing build and a
# variant timing build tools/gpu/ab/$1.so
mkdir -p gpurun_out
for v in base $1; do
  lib=tools/gpu/libpsim_timing.so; [ "$v" != base ] && lib=tools/gpu/ab/$v.so
  PSIM_LIB=$lib PSIM_DEBUG_TIMING=900 PSIM_DEBUG_TIMING_OUT=gpurun_out/timing_e8_$v.txt timeout 600 python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu --emulate-rank 0/8 2>&1 | tail -1 | cut -c1-50
  PSIM_LIB=$lib PSIM_DEBUG_TIMING=900 PSIM_DEBUG_TIMING_OUT=gpurun_out/timing_900_$v.txt timeout 600 python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu 2>&1 | tail -1 | cut -c1-50
done
