# e2e (pinned host trace streamed by the loader) with 1 / 2 / 3 cohorts, config 3
for r in 1 2; do for c in 1 2 3; do
  PSIM_COHORTS=$c timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('cohorts $c run $r value', round(d['value'],1), 'e2e', round(d['e2e']['value'],1))"
done; done
