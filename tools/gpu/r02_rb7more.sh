# RB7 tests incl. the many-tiles-per-CTA parity case, then config 5 at 1B rows with the corrected roofline label
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_rb7.py -q -m gpu -s > gpurun_out/rb7_tests.log 2>&1; echo "rb7 tests rc=$?"; tail -3 gpurun_out/rb7_tests.log
timeout 1500 python bench.py --config c5 --steps 1 --warmup 1 --no-cpu --no-e2e > gpurun_out/ev_bench_c5_1B_b.json 2> gpurun_out/ev_bench_c5_1B_b.log; echo "c5 rc=$?"
