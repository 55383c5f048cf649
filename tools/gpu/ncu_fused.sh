# ncu evidence for the fused path: launch list + full captures of both kernels (c3 batch shape)
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 200 -c 60 --kill on --csv \
  --log-file gpurun_out/launches_fused_c3p.csv python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_list.log 2>&1
echo "list rc=$?"
for k in conv_stack_kernel fc1_head_kernel; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 150 -c 1 --kill on \
  -o gpurun_out/prof_fused_$k python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_$k.log 2>&1
echo "$k rc=$?"
done
timeout 300 python -m pytest tests -x -q -m "gpu" -k "fused_full" 2>&1 | tail -5
