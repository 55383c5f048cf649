# full GPU suite + bench line
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/gpu_tests.log
timeout 600 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.log; echo "bench rc=$?"
python -c "import json; d=json.load(open('gpurun_out/bench_c3.json')); r=d['roofline']; print('VALUE', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'ms', round(d['ms_per_step'],1), r['frac'], {k: v['ms'] for k, v in r['kernels'].items()})"
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
