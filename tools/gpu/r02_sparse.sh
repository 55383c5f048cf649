# 2:4 sparse path: metadata probe (id2 alternation), GPU parity tests, layer-wise dense vs sparse bench
mkdir -p gpurun_out
bash tools/gpu/sparse_probe.sh > gpurun_out/sparse_probe3.log 2>&1
timeout 900 python -m pytest tests/test_gpu_sparse.py -q -m gpu -x -s > gpurun_out/r02_sparse_tests.log 2>&1; echo "sparse tests rc=$?"; grep -E "S2 sparse|S3 sparse|passed|failed" gpurun_out/r02_sparse_tests.log | tail -8
for v in "--layerwise" "--sparse"; do
  timeout 600 python bench.py --steps 2 --warmup 1 --no-cpu --no-e2e $v > gpurun_out/r02_bench_c3$v.json 2> gpurun_out/r02_bench_c3$v.err; echo "bench $v rc=$?"
  python -c "
import json; d=json.load(open('gpurun_out/r02_bench_c3$v.json')); r=d['roofline']; print('$v VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1), {k:v['ms'] for k,v in r['kernels'].items()})"
done
