# A/B of environment settings of one build on one box (alternating runs): G = 1, the G = 4 and
# G = 8 slices.  Usage: bash tools/gpu/abe.sh "VAR=0 VAR=1" [lib]
V="$1"; LIB="${2:-paper_conf_sc_pandeylfhl22_b200/libpsim.so}"
for g in 1 4 8; do for r in 1 2; do for v in $V; do
  emu=""; st="--steps 5"; [ $g -gt 1 ] && emu="--emulate-rank 0/$g" && st="--steps 3"
  env $v PSIM_LIB=$LIB timeout 300 python bench.py $st --warmup 3 --no-cpu --no-e2e $emu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v G=$g run $r', round(d['value'],1), d['total_cycles'], {k:v['ms'] for k,v in r['kernels'].items()})"
done; done; done
