# fused-path parity subset + a bench line
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu -k "s1_teacher or residency or s3_c3_small or fused_full or pec_s1_fused or metrics_fused or smoke" > gpurun_out/fast.log 2>&1; echo "fast rc=$?"; tail -15 gpurun_out/fast.log
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_fast.json 2> gpurun_out/bench_fast.log; echo "bench rc=$?"
python -c "import json; d=json.load(open('gpurun_out/bench_fast.json')); r=d['roofline']; print('VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1), r['frac'], {k: v['ms'] for k, v in r['kernels'].items()})"
