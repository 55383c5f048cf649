# PDL on/off x cohorts with SM shares at the G = 8 slice (and G = 1)
for g in 8 1; do for cfg in "1 0 0" "1 0 1" "2 1 0" "2 1 1" "4 1 1"; do set -- $cfg
  emu=""; [ $g -gt 1 ] && emu="--emulate-rank 0/$g"
  PSIM_COHORTS=$1 PSIM_COHORT_SMS=$2 PSIM_NO_PDL=$3 timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e $emu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('G=$g cohorts=$1 sms=$2 nopdl=$3 VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1))"
done; done
