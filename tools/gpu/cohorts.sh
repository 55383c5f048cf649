# cohort sweep: GPU tests (default cohorts), bench at G=1 for PSIM_COHORTS=1,2,3,4, emulated shares
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x -k "fused or c3 or smoke or metrics or pec or residency" > gpurun_out/iter_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/iter_tests.log
for c in 1 2 3 4; do
PSIM_COHORTS=$c timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/coh_$c.json 2> gpurun_out/coh_$c.log; echo "bench c=$c rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/coh_$c.json')); r=d['roofline']; print('COH $c VALUE', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'ms', round(d['ms_per_step'],1), r['frac'], {k:v['ms'] for k,v in r['kernels'].items()})"
done
for g in 2 8; do for c in 1 2 4; do
PSIM_COHORTS=$c timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --emulate-rank 0/$g 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('G=$g coh=$c per-GPU', round(d['value'],1), 'ms', round(d['ms_per_step'],1))"
done; done
