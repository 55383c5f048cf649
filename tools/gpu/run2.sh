# full GPU tests (not slow) + bench c2/c3 timing
timeout 900 python -m pytest tests -x -q -m "gpu and not slow" 2>&1 | tail -15
timeout 600 python bench.py --config c2 --steps 2 --warmup 1 --cpu-budget 5 2>&1 | tail -3
timeout 900 python bench.py --config c3 --steps 2 --warmup 1 --cpu-budget 5 --no-e2e 2>&1 | tail -3
