O=gpurun_out; T=e4
python -c "import __graft_entry__ as g; g.build()" > $O/build_$T.log 2>&1 || { tail -5 $O/build_$T.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -m gpu -q -x > $O/pytest_$T.log 2>&1; tail -3 $O/pytest_$T.log
run() { n=$1; shift; timeout 600 python bench.py --no-e2e --no-cpu --reps 2 "$@" > $O/bench_${T}_$n.json 2> $O/bench_${T}_$n.err; python - $O/bench_${T}_$n.json $n <<'PY'
import json,sys
try:
    d=json.load(open(sys.argv[1]))
    ph=d['phases_ms_per_step']
    print(sys.argv[2], 'val %.2f G'%(d['value']/1e9), 'ms %.3f'%d['ms_per_step'], 'pmd %.3f'%ph['push_move_deposit'], 'cont %.3f'%ph.get('continue',0), 'seg %.3f'%ph.get('segred',0), 'fill %.3f'%ph.get('fill',0), 'sortmove %.3f'%ph.get('sort_move',0), 'frac %.3f'%d['roofline']['frac'], 'hops %.3f'%d['walk']['hops_per_particle_last_step'])
except Exception as e: print(sys.argv[2], 'FAILED', e)
PY
}
for cfg in c2 c4; do
  run ${cfg}_full --config $cfg
  for v in L1 L2 L3 L4 q; do OPP_LIB=variants/libopp_$v.so run ${cfg}_$v --config $cfg; done
done
for d in 0 1 2; do run c5_dep$d --config c5 --deposit $d --steps 10; done
run c2_dep2 --config c2 --deposit 2
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 4 -c 1 -o $O/prof_${T}_c4 python bench.py --steps 2 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-full $?
OPP_LIB=variants/libopp_q.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 4 -c 1 -o $O/prof_${T}_c2q python bench.py --config c2 --steps 2 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-full $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 4 -c 1 -o $O/prof_${T}_c2 python bench.py --config c2 --steps 2 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-full $?
