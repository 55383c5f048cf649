# per variant: fused-path parity subset + bench line (usage: bash variants3.sh A SPLIT ...)
B=paper_conf_sc_pandeylfhl22_b200
mkdir -p gpurun_out
for v in "$@"; do
cp tools/gpu/lib$v.so $B/libpsim.so
timeout 900 python -m pytest tests -x -q -m gpu -k "residency or s3_c3_small or fused_full or pec_s1_fused or metrics_fused" > gpurun_out/var_$v.log 2>&1; echo "$v tests rc=$? $(tail -1 gpurun_out/var_$v.log)"
timeout 600 python bench.py --config c3 --steps 3 --warmup 3 --no-cpu --no-e2e 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1), r['frac'], {k: v['ms'] for k, v in r['kernels'].items()})"
done
cp tools/gpu/libA.so $B/libpsim.so
