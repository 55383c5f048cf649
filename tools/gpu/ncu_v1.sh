# ncu evidence for the v1 (layer-by-layer) path on config 3
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s 11460 -c 2300 --csv \
  --log-file gpurun_out/launches_v1_c3.csv python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --cpu-budget 1 > gpurun_out/ncu_list.log 2>&1
echo "list rc=$?"
for k in gather_kernel gemm_tc_kernel update_kernel; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 300 -c 2 \
  -o gpurun_out/prof_v1_$k python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --cpu-budget 1 > gpurun_out/ncu_$k.log 2>&1
echo "$k rc=$?"
done
ls -la gpurun_out
