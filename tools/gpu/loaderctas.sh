# e2e (pinned host trace, streamed) vs the zero-copy loader's grid cap and the cohort count
for coh in 1 2; do for c in 64 296; do
PSIM_COHORTS=$coh PSIM_LOADER_CTAS=$c timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('cohorts $coh loader CTAs $c VALUE', round(d['value'],1), 'e2e', round(d['e2e']['value'],1))"
done; done
