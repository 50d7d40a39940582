set -x
TAG=$1
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
for v in "--sort 0" "--sort 1" "--sort 2" "--sort 5" "--sort 2 --deposit 1" "--sort 5 --deposit 1" "--sort 2 --hpass 2" "--sort 2 --hpass 8"; do
  echo "== $v"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu $v 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value']/1e9, d['ms_per_step'], d['roofline']['frac'], json.dumps(d['phases_ms_per_step']))"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 2 -c 1 -o gpurun_out/prof_pmd_$TAG python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --sort 2 > gpurun_out/ncu_full_$TAG.log 2>&1; echo ncu2 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sort_scatter -s 3 -c 1 -o gpurun_out/prof_sort_$TAG python bench.py --steps 4 --warmup 1 --no-e2e --no-cpu --sort 1 > /dev/null 2>&1; echo ncu3 $?
