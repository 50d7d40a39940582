# usage: bash scripts/gpu_sweep.sh TAG  -- parity tests + bench variants + ncu of the best
set -x
TAG=$1
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
for v in "--sort 0" "--sort 1" "--sort 2" "--sort 5" "--sort 10" "--sort 2 --deposit 1" "--sort 5 --deposit 1" "--sort 2 --deposit 2" "--sort 2 --dh"; do
  echo "== $v"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu $v 2>&1 | tail -1
done
timeout 600 python bench.py --steps 20 --warmup 3 --sort 2 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 4 --warmup 1 --no-e2e --no-cpu --sort 2 > /dev/null 2>&1; echo ncu1 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit -s 4 -c 1 -o gpurun_out/prof_pmd_$TAG python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --sort 2 > gpurun_out/ncu_full_$TAG.log 2>&1; echo ncu2 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sort_scatter -s 1 -c 1 -o gpurun_out/prof_sort_$TAG python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --sort 1 > /dev/null 2>&1; echo ncu3 $?
