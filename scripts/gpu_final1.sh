set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/bench_final1.json 2> gpurun_out/bench_final1.err; tail -3 gpurun_out/bench_final1.err; cat gpurun_out/bench_final1.json
timeout 900 python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/bench_ref1.json 2>&1; tail -1 gpurun_out/bench_ref1.json
for d in 0 1 2; do timeout 600 python bench.py --config c5 --deposit $d --no-e2e --no-cpu --steps 10 > gpurun_out/bench_c5_dep$d.json 2>&1; tail -1 gpurun_out/bench_c5_dep$d.json | cut -c1-400; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_final1.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu1 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 6 -c 1 -o gpurun_out/prof_final1 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu2 $?
