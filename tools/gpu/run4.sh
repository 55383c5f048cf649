timeout 300 python -m pytest tests -x -q -m "gpu" -k "s3_c3_small or fused_full or smoke or s1_hand" 2>&1 | tail -25
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -2
timeout 600 python bench.py --config c3 --steps 2 --warmup 1 --cpu-budget 3 --no-e2e 2>&1 | tail -2
