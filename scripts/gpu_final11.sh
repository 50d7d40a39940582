# Session measurement (11th pass: end of session, C3 e2e overlap): tests, smoke, C2 + reference, C3 + reference, C5 modes, ncu launch lists + full captures
# reference arm, C5 deposit modes, ncu launch lists + full captures of pass 1 (C2) and k_em_move_deposit (C3)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv,noheader
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_f11.log 2>&1; tail -2 gpurun_out/pytest_gpu_f11.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_f11.json 2> gpurun_out/bench_f11.err; tail -2 gpurun_out/bench_f11.err; cut -c1-200 gpurun_out/bench_f11.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref_f11.json 2>&1; tail -1 gpurun_out/bench_ref_f11.json | cut -c1-200
timeout 600 python bench.py --config c3 > gpurun_out/bench_c3_f11.json 2> gpurun_out/bench_c3_f11.err; cut -c1-200 gpurun_out/bench_c3_f11.json
timeout 600 python bench.py --config c3 --impl reference --steps 5 --warmup 1 > gpurun_out/bench_c3_ref_f11.json 2>&1; tail -1 gpurun_out/bench_c3_ref_f11.json | cut -c1-200
for d in 0 1 2; do timeout 600 python bench.py --config c5 --deposit $d --no-e2e --no-cpu --steps 10 > gpurun_out/bench_c5_f11_dep$d.json 2>&1; tail -1 gpurun_out/bench_c5_f11_dep$d.json | cut -c1-160; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_f11.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu1 $?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3_f11.csv python bench.py --config c3 --steps 5 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu2 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 6 -c 1 -o gpurun_out/prof_f11 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu3 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_em_move_deposit -s 3 -c 1 -o gpurun_out/prof_f11_em python bench.py --config c3 --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu4 $?
timeout 600 python bench.py --field-model boltzmann --no-cpu > gpurun_out/bench_boltz_f11.json 2> gpurun_out/bench_boltz_f11.err; cut -c1-200 gpurun_out/bench_boltz_f11.json
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_newton_eval -s 2 -c 1 -o gpurun_out/prof_f11_newton python bench.py --field-model boltzmann --steps 2 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu5 $?
