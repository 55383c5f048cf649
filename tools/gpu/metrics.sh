# interval-metrics parity + full GPU suite + a bench line (metrics off) to check for regressions
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_metrics.py -x -q > gpurun_out/metrics_tests.log 2>&1; echo "metrics rc=$?"; tail -15 gpurun_out/metrics_tests.log
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/gpu_tests.log
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.log; echo "bench rc=$?"
python -c "import json; d=json.load(open('gpurun_out/bench_c3.json')); print('VALUE', d['value'], d['e2e']['value'], d['roofline']['frac'])"
