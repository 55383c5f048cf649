# bench each tools/gpu/lib<V>.so variant given as arguments, then the timing lib
mkdir -p gpurun_out
B=paper_conf_sc_pandeylfhl22_b200
for v in "$@"; do
cp tools/gpu/lib$v.so $B/libpsim.so
timeout 600 python bench.py --config c3 --steps 2 --warmup 1 --no-cpu --no-e2e 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1), r['frac'], {k: v['ms'] for k, v in r['kernels'].items()})"
done
cp tools/gpu/lib$1.so $B/libpsim.so
timeout 900 python -m pytest tests -x -q -m "gpu" -k "s1_teacher or residency or s3_c3_small or fused_full or pec_s1_fused" 2>&1 | tail -2
cp tools/gpu/libpsim_timing.so $B/libpsim.so
PSIM_DEBUG_TIMING=900 PSIM_DEBUG_TIMING_OUT=gpurun_out/timing_900.txt timeout 600 python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu 2>&1 | tail -1 | cut -c1-50
