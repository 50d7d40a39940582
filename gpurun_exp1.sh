O=gpurun_out; T=e1
python -c "import __graft_entry__ as g; g.build()" > $O/build_$T.log 2>&1 || { tail -5 $O/build_$T.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -m gpu -q -x > $O/pytest_$T.log 2>&1; tail -2 $O/pytest_$T.log
run() { n=$1; shift; timeout 600 python bench.py --no-e2e --no-cpu --reps 2 "$@" > $O/bench_${T}_$n.json 2> $O/bench_${T}_$n.err; python - $O/bench_${T}_$n.json $n <<'PY'
import json,sys
try:
    d=json.load(open(sys.argv[1]))
    ph=d['phases_ms_per_step']
    print(sys.argv[2], 'val %.2f G'%(d['value']/1e9), 'ms %.3f'%d['ms_per_step'], 'pmd %.3f'%ph['push_move_deposit'], 'fill %.3f'%ph.get('fill',0), 'sortmove %.3f'%ph.get('sort_move',0), 'frac %.3f'%d['roofline']['frac'], 'hops %.3f'%d['walk']['hops_per_particle_last_step'])
except Exception as e: print(sys.argv[2], 'FAILED', e)
PY
}
run c4_q
OPP_LIB=variants/libopp_noq.so run c4_noq
run c4_s0 --sort 0 --sort-init 1
run c4_s25 --sort 25 --steps 25
run c4_s50 --sort 50 --steps 25
run c4_ov25 --ov 0.25
run c4_mh --mh
run c2_q --config c2
OPP_LIB=variants/libopp_noq.so run c2_noq --config c2
