mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sparse.py -q -m gpu -s > gpurun_out/r02_sparse_tests.log 2>&1; echo "sparse tests rc=$?"; grep -E "S2 sparse|S3 sparse|passed|failed" gpurun_out/r02_sparse_tests.log | tail -8
for v in "--layerwise" "--sparse"; do
  timeout 600 python bench.py --steps 2 --warmup 1 --no-cpu --no-e2e $v > gpurun_out/r02_bench_c3$v.json 2> gpurun_out/r02_bench_c3$v.err; echo "bench $v rc=$?"
  python -c "
import json; d=json.load(open('gpurun_out/r02_bench_c3$v.json')); r=d['roofline']; print('$v VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1), {k:v['ms'] for k,v in r['kernels'].items()})"
done
# ncu: tensor-pipe time of the dense vs sparse conv3/fc1 GEMMs (one launch each, config-3 batch shape)
for v in "--layerwise" "--sparse"; do
  timeout 600 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__inst_executed_pipe_tensor.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:gemm -s 40 -c 8 --csv \
    python bench.py --config c3p --steps 1 --warmup 0 --no-cpu --no-e2e $v > gpurun_out/r02_ncu_gemm$v.csv 2> /dev/null; echo "ncu $v rc=$?"
done
