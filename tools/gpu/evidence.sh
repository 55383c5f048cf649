# Round evidence: bench line (default), reference arm, ncu launch list + full captures, smoke.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_info.csv
timeout 900 python bench.py > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.log; echo "bench rc=$?"
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.log; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 200 -c 60 --kill on --csv \
  --log-file gpurun_out/launches_c3p.csv python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_list.log 2>&1; echo "list rc=$?"
for k in conv_stack_kernel fc1_head_kernel; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 150 -c 1 --kill on \
  -o gpurun_out/prof_$k python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_$k.log 2>&1
echo "$k rc=$?"
done
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
