# e2e (pinned host trace, streaming loader) of builds tools/gpu/ab/<v>.so, config 3, alternating
for r in 1 2 3; do for v in $1; do
  PSIM_LIB=tools/gpu/ab/$v.so timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$v run $r value', round(d['value'],1), 'e2e', round(d['e2e']['value'],1))"
done; done
