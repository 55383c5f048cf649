mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_stack -s 150 -c 1 --kill on \
  -o gpurun_out/prof_conv_stack_g4 python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_cs.log 2>&1
echo "rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fc1_head -s 150 -c 1 --kill on \
  -o gpurun_out/prof_fc1_head_g4 python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_fh.log 2>&1
echo "rc=$?"
