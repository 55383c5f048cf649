mkdir -p gpurun_out
cp tools/gpu/libA.so paper_conf_sc_pandeylfhl22_b200/libpsim.so
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_stack_kernel -s 120 -c 1 --kill on \
  -o gpurun_out/prof_conv_A python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_conv_A.log 2>&1
echo "rc=$?"
