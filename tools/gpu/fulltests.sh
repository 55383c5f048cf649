timeout 1500 python -m pytest tests -q -m "gpu" --durations=5 2>&1 | tail -12
