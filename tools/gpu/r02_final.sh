# Round-2 final evidence: r02_evidence.sh (suite, smoke, bench, reference arm, emulated
# ranks, ncu list + full captures), then config 5 at full size (1B rows, 262144 sub-traces,
# RB7; device-resident and e2e from a pinned host trace).
bash tools/gpu/r02_evidence.sh
timeout 1500 python bench.py --config c5 --steps 1 --warmup 1 --no-cpu --no-e2e > gpurun_out/ev_bench_c5_1B.json 2> gpurun_out/ev_bench_c5_1B.log; echo "c5 rc=$?"
timeout 1500 python bench.py --config c5 --steps 1 --warmup 1 --no-cpu > gpurun_out/ev_bench_c5_1B_e2e.json 2> gpurun_out/ev_bench_c5_1B_e2e.log; echo "c5 e2e rc=$?"
