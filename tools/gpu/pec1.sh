set -x
nvidia-smi --query-gpu=name --format=csv,noheader
timeout 1200 python -m pytest tests/test_gpu_pec.py -x -q 2>&1 | tail -25
timeout 900 python -m pytest tests -x -q -m "gpu" -k "s1_teacher or s1_hand or residency or s3_c3_small" 2>&1 | tail -3
