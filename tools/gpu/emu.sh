# per-GPU throughput at G GPUs, emulated on one GPU (rank 0's share, no NCCL)
mkdir -p gpurun_out
for g in 2 4 8; do
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --emulate-rank 0/$g 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('G=$g per-GPU VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1), 'x$g =', round($g*d['value'],1))"
done
