# ncu --set full with source correlation of conv_stack (config-3 batch shape, step 150)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-conv_stack} -s 150 -c 1 --kill on \
  -o gpurun_out/prof_${KNAME:-conv}_src python bench.py --config c3p --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_src.log 2>&1
echo "ncu rc=$?"
