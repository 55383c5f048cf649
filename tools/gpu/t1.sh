mkdir -p gpurun_out
cp tools/gpu/libA.so paper_conf_sc_pandeylfhl22_b200/libpsim.so
timeout 900 python -m pytest tests -x -q -m "gpu" -k "s1_teacher or residency or s3_c3_small or fused_full or pec_s1_fused" > gpurun_out/t1.log 2>&1
tail -5 gpurun_out/t1.log
