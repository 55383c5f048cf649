# one optimisation iteration (round 2): fused-path parity tests, bench line, timeline
# (timing build tools/gpu/libpsim_timing.so), per-GPU share at G = 8
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "fused or s1 or c3_small or deterministic or residency" > gpurun_out/iter_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/iter_tests.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/iter_bench.json 2> gpurun_out/iter_bench.log; echo "bench rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/iter_bench.json')); r=d['roofline']; print('VALUE', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'ms', round(d['ms_per_step'],1), r['frac'], r['step']['frac'], {k:v['ms'] for k,v in r['kernels'].items()})"
bash tools/gpu/timing6.sh > /dev/null 2>&1
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --emulate-rank 0/8 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('G=8 per-GPU VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1), {k:v['ms'] for k,v in r['kernels'].items()})"
