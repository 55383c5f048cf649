# A/B/... of tools/gpu/ab/<name>.so builds on one box (alternating runs), G = 1 and the G = 8
# slice (bench.py --emulate-rank 0/8).  Usage: bash tools/gpu/abn.sh "A pf8 pf16" [G=1 rounds] [G=8 rounds]
V="$1"; R1="${2:-2}"; R8="${3:-2}"
for r in $(seq 1 $R1); do for v in $V; do
  PSIM_LIB=tools/gpu/ab/$v.so timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v G=1 run $r', round(d['value'],1), d['total_cycles'], {k:v['ms'] for k,v in r['kernels'].items()})"
done; done
for r in $(seq 1 $R8); do for v in $V; do
  PSIM_LIB=tools/gpu/ab/$v.so timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --emulate-rank 0/8 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v G=8 run $r', round(d['value'],1), d['total_cycles'], {k:v['ms'] for k,v in r['kernels'].items()})"
done; done
