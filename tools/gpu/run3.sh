timeout 1500 python -m pytest tests -q -m "gpu" -x --durations=8 2>&1 | tail -25
