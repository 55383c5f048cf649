mkdir -p gpurun_out
cp paper_conf_sc_pandeylfhl22_b200/libpsim.so /tmp/libpsim_prod.so
cp tools/gpu/libpsim_timing.so paper_conf_sc_pandeylfhl22_b200/libpsim.so
PSIM_DEBUG_TIMING=900 PSIM_DEBUG_TIMING_OUT=gpurun_out/timing_e8.txt timeout 600 python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu --emulate-rank 0/8 2>&1 | tail -1 | cut -c1-50
PSIM_DEBUG_TIMING=900 PSIM_DEBUG_TIMING_OUT=gpurun_out/timing_900.txt timeout 600 python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu 2>&1 | tail -1 | cut -c1-50
cp /tmp/libpsim_prod.so paper_conf_sc_pandeylfhl22_b200/libpsim.so
