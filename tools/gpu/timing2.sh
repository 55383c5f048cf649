mkdir -p gpurun_out
PSIM_DEBUG_TIMING=150 PSIM_DEBUG_TIMING_OUT=gpurun_out/conv_timing.txt timeout 600 python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu 2>&1 | tail -1 | cut -c1-100
