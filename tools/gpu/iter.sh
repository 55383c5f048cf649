# one iteration: fused-path GPU parity tests, bench line, timeline (timing build), per-GPU shares
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x -k "fused or c3 or smoke or metrics or pec" > gpurun_out/iter_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/iter_tests.log
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/iter_bench.json 2> gpurun_out/iter_bench.log; echo "bench rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/iter_bench.json')); r=d['roofline']; print('VALUE', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'ms', round(d['ms_per_step'],1), r['frac'], {k:v['ms'] for k,v in r['kernels'].items()})"
bash tools/gpu/timing6.sh > /dev/null 2>&1
bash tools/gpu/emu.sh
