# config-4 sweep (N 256..262144 x W 0/128/1000/10000) + S4 geometry, against the cached unpartitioned oracle
mkdir -p gpurun_out
timeout 3000 python tools/accuracy.py --config4 --out gpurun_out/r02_config4_sweep.json > gpurun_out/r02_config4_sweep.log 2>&1; echo "config4 rc=$?"
