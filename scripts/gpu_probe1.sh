# L1 data-pipe costs of the building blocks, and a source-level ncu capture of pass 1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 120 scripts/micro/wf_cost > gpurun_out/wf_cost.txt 2>&1; echo wf $?
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --field 0 > gpurun_out/bench_p1.json 2> gpurun_out/bench_p1.err; echo bench $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 6 -c 1 -o gpurun_out/prof_src python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu --field 0 > /dev/null 2>&1; echo ncu $?
