# End-of-session measurement: tests, smoke, bench (default = C2 with field solve), reference arm,
# ncu launch list + full capture of pass 1 and of the CG kernel
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv,noheader
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_f2.log 2>&1; tail -2 gpurun_out/pytest_gpu_f2.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_f2.json 2> gpurun_out/bench_f2.err; tail -2 gpurun_out/bench_f2.err; cat gpurun_out/bench_f2.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref_f2.json 2>&1; tail -1 gpurun_out/bench_ref_f2.json | cut -c1-300
timeout 600 python bench.py --field 0 --dhmode 2 --no-e2e --no-cpu --steps 20 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('dhmode2', round(d['value']/1e9,2), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit',)})"
for d in 0 1 2; do timeout 600 python bench.py --config c5 --deposit $d --no-e2e --no-cpu --steps 10 > gpurun_out/bench_c5_f2_dep$d.json 2>&1; tail -1 gpurun_out/bench_c5_f2_dep$d.json | cut -c1-200; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_f2.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu1 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 6 -c 1 -o gpurun_out/prof_f2 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu2 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pcg -s 4 -c 1 -o gpurun_out/prof_f2_cg python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu3 $?
