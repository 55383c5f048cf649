# ncu --set full with source correlation of one fc1_head launch of the G = 8 slice (step 900)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-fc1_head} -s 900 -c 1 --kill on \
  -o gpurun_out/prof_${KNAME:-fc1}_e8_src python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu --emulate-rank 0/8 > gpurun_out/ncu_src_e8.log 2>&1
echo "ncu rc=$?"
