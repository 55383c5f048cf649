set -x
timeout 900 python tools/accuracy.py --L 200000 2>&1 | tail -30
mkdir -p gpurun_out; cp profiles/r01_accuracy.json gpurun_out/ 2>/dev/null
for c in 0 100; do
timeout 900 python bench.py --config c3 --steps 2 --warmup 1 --no-cpu --no-e2e --correction $c 2>&1 | tail -1 > gpurun_out/bench_pec$c.json
python -c "
import json; d=json.load(open('gpurun_out/bench_pec$c.json')); print('CORR $c VALUE', round(d['value'],1), d['total_cycles'], d['stats'])"
done
