mkdir -p gpurun_out
cp paper_conf_sc_pandeylfhl22_b200/libpsim.so /tmp/libpsim_prod.so
cp tools/gpu/libpsim_timing.so paper_conf_sc_pandeylfhl22_b200/libpsim.so
for s in 300 900; do
PSIM_DEBUG_TIMING=$s PSIM_DEBUG_TIMING_OUT=gpurun_out/timing_$s.txt timeout 600 python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu 2>&1 | tail -1 | cut -c1-50
done
cp /tmp/libpsim_prod.so paper_conf_sc_pandeylfhl22_b200/libpsim.so
