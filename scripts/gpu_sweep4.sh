set -x
TAG=$1
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
for v in "--sort 0" "--sort 0 --direct" "--sort 5" "--sort 10" "--sort 5 --deposit 1" "--sort 0 --hpass 16"; do
  echo "== $v"; timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu $v 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})"
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 2 -c 1 -o gpurun_out/prof_pmd_$TAG python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --sort 0 > gpurun_out/ncu_full_$TAG.log 2>&1; echo ncu2 $?
