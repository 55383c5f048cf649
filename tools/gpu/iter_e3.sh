# conv3 epilogue split over EG-A / EG-B: fused-path parity, then A/B
set -x
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "fused or pair or s3_c3 or config3 or s1" 2>&1 | tail -3
bash tools/gpu/ab.sh
for v in A B; do
  PSIM_LIB=tools/gpu/ab/$v.so timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e --emulate-rank 0/4 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$v G=4 VALUE', round(d['value'],1))"
done
