O=gpurun_out; T=e2
python -c "import __graft_entry__ as g; g.build()" > $O/build_$T.log 2>&1 || { tail -5 $O/build_$T.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py tests/test_gpu_sanitize.py -m gpu -q -x > $O/pytest_$T.log 2>&1; tail -3 $O/pytest_$T.log
run() { n=$1; shift; timeout 600 python bench.py --no-e2e --no-cpu --reps 2 "$@" > $O/bench_${T}_$n.json 2> $O/bench_${T}_$n.err; python - $O/bench_${T}_$n.json $n <<'PY'
import json,sys
try:
    d=json.load(open(sys.argv[1]))
    ph=d['phases_ms_per_step']
    print(sys.argv[2], 'val %.2f G'%(d['value']/1e9), 'ms %.3f'%d['ms_per_step'], 'pmd %.3f'%ph['push_move_deposit'], 'fill %.3f'%ph.get('fill',0), 'sortmove %.3f'%ph.get('sort_move',0), 'frac %.3f'%d['roofline']['frac'], 'hops %.3f'%d['walk']['hops_per_particle_last_step'])
except Exception as e: print(sys.argv[2], 'FAILED', e)
PY
}
run c2_aux --config c2
OPP_LIB=variants/libopp_noaux.so run c2_noaux --config c2
OPP_LIB=variants/libopp_auxq.so run c2_auxq --config c2
run c4_aux
OPP_LIB=variants/libopp_noaux.so run c4_noaux
OPP_LIB=variants/libopp_auxq.so run c4_auxq
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 6 -c 1 -o $O/prof_$T python bench.py --config c2 --steps 2 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-full $?
