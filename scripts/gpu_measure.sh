#!/bin/bash
# The measurement pass of a round (run under gpurun from the repo root):
#   TAG=r02a STAGES="tests bench c2 empty c5 c3 loopback ncu" scripts/gpu_measure.sh
# then, here: scripts/ncu_summary.py traffic gpurun_out/prof_c4_$TAG.ncu-rep c4_dep1_dh1 prof_c4_$TAG
# Every output lands in gpurun_out/ (summaries are copied to profiles/ by hand).
TAG=${TAG:-r02}
STAGES=${STAGES:-"tests bench c2 c5 c3 ncu"}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -5 $O/build_$TAG.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,memory.total --format=csv,noheader
has() { [[ " $STAGES " == *" $1 "* ]]; }
if has tests; then
  timeout 1800 python -m pytest tests -m gpu -q -x > $O/pytest_gpu_$TAG.log 2>&1; tail -3 $O/pytest_gpu_$TAG.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
fi
if has bench; then
  timeout 1200 python bench.py > $O/bench_c4_$TAG.json 2> $O/bench_c4_$TAG.err; tail -3 $O/bench_c4_$TAG.err; cut -c1-300 $O/bench_c4_$TAG.json
  timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_c4_ref_$TAG.json 2>&1; tail -1 $O/bench_c4_ref_$TAG.json | cut -c1-200
fi
if has c2; then
  timeout 900 python bench.py --config c2 > $O/bench_c2_$TAG.json 2> $O/bench_c2_$TAG.err; tail -2 $O/bench_c2_$TAG.err; cut -c1-300 $O/bench_c2_$TAG.json
fi
if has c5; then
  for d in 0 1 2; do timeout 600 python bench.py --config c5 --deposit $d --no-e2e --no-cpu --steps 10 --reps 1 > $O/bench_c5_${TAG}_dep$d.json 2>&1; tail -1 $O/bench_c5_${TAG}_dep$d.json | cut -c1-160; done
fi
if has empty; then
  timeout 900 python bench.py --config c2 --empty --steps 200 --reps 1 > $O/bench_c2_empty_$TAG.json 2> $O/bench_c2_empty_$TAG.err; tail -2 $O/bench_c2_empty_$TAG.err; cut -c1-200 $O/bench_c2_empty_$TAG.json
fi
if has c3; then
  timeout 600 python bench.py --config c3 > $O/bench_c3_$TAG.json 2> $O/bench_c3_$TAG.err; cut -c1-200 $O/bench_c3_$TAG.json
fi
if has loopback; then
  timeout 900 python bench.py --gpus 2 --loopback --n0 200000000 --no-cpu > $O/bench_c4_loop2_$TAG.json 2> $O/bench_c4_loop2_$TAG.err; tail -2 $O/bench_c4_loop2_$TAG.err; cut -c1-300 $O/bench_c4_loop2_$TAG.json
fi
if has ncu; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_c4_$TAG.csv python bench.py --steps 10 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-launches $?
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 5 -c 1 -o $O/prof_c4_$TAG python bench.py --steps 2 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-full $?
fi
if has ncu2; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 5 -c 1 -o $O/prof_c2_$TAG python bench.py --config c2 --steps 2 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-full-c2 $?
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_em_move_deposit -s 4 -c 1 -o $O/prof_c3_$TAG python bench.py --config c3 --steps 2 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-full-c3 $?
fi
