# RB7 parity + full GPU suite
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_rb7.py -x -q > gpurun_out/rb7_tests.log 2>&1; echo "rb7 rc=$?"; tail -25 gpurun_out/rb7_tests.log
timeout 2400 python -m pytest tests -q -m gpu -x > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/gpu_tests.log
