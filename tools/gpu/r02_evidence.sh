# Round-2 evidence: full GPU suite + smoke, bench line (driver settings), reference arm,
# emulated per-GPU shares at G = 2/4/8, ncu launch list + full captures (with source) of
# both fused kernels.  Summaries are made on the CPU side (tools/ncu_summary.py,
# tools/ncu_src_summary.py) and copied into profiles/.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv > gpurun_out/ev_gpu_info.csv
timeout 2400 python -m pytest tests -q -m gpu -s > gpurun_out/ev_gpu_tests.log 2>&1; echo "gpu tests rc=$?"; tail -2 gpurun_out/ev_gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/ev_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/ev_smoke.log
timeout 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/ev_bench_c3.json 2> gpurun_out/ev_bench_c3.log; echo "bench rc=$?"
timeout 900 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/ev_bench_ref.json 2> gpurun_out/ev_bench_ref.log; echo "ref rc=$?"
for g in 2 4 8; do
  timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --emulate-rank 0/$g > gpurun_out/ev_emu_$g.json 2>/dev/null; echo "emu $g rc=$?"
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 200 -c 60 --kill on --csv \
  --log-file gpurun_out/ev_launches_c3p.csv python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ev_ncu_list.log 2>&1; echo "list rc=$?"
for k in conv_stack_kernel fc1_head_kernel; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 150 -c 1 --kill on \
    -o gpurun_out/ev_prof_$k python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ev_ncu_$k.log 2>&1
  echo "$k rc=$?"
done
