# full GPU test suite + round evidence (bench line, reference arm, ncu launch list + full captures, smoke)
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/gpu_tests.log
bash tools/gpu/evidence.sh
