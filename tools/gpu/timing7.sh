# PSIM_TIMING timelines of the current code (CTA 0, step 900): G = 8 slice and G = 1
mkdir -p gpurun_out
for e in 8 1; do
  PSIM_LIB=tools/gpu/libpsim_timing.so PSIM_DEBUG_TIMING=900 PSIM_DEBUG_TIMING_OUT=gpurun_out/timing7_g$e.txt timeout 600 \
    python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu --emulate-rank 0/$e 2>&1 | tail -1 | cut -c1-60
done
