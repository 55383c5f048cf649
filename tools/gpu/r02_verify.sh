# full GPU suite + smoke + a short bench at HEAD (after the CNN error-path fix)
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/verify_gpu_tests.log 2>&1; echo "gpu tests rc=$?"; tail -2 gpurun_out/verify_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('bench', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'frac', d['roofline']['frac'], d['clocks'])"
