set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
nproc; free -g | head -2
python -c "import torch;print(torch.cuda.get_device_name())"
timeout 600 python -m pytest tests -x -q -m "gpu and not slow" -k "s1 or state_machine" 2>&1 | tail -30
timeout 300 python -m pytest tests -x -q -m "gpu and not slow" -k "s2" 2>&1 | tail -30
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -5
