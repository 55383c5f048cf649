# fast lib: tests + bench; then timing lib: per-stage timestamps
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m "gpu" -k "s1 or s3_c3_small or fused_full or state_machine" 2>&1 | tail -2
timeout 600 python bench.py --config c3 --steps 2 --warmup 1 --no-e2e --no-cpu 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('VALUE', d['value'], 'ms', d['ms_per_step'], r['kernel'], r['frac'], r['kernels'])"
cp tools/gpu/libpsim_timing.so paper_conf_sc_pandeylfhl22_b200/libpsim.so
PSIM_DEBUG_TIMING=150 PSIM_DEBUG_TIMING_OUT=gpurun_out/conv_timing.txt timeout 600 python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu 2>&1 | tail -1 | cut -c1-100
