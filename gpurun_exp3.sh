O=gpurun_out; T=e3
python -c "import __graft_entry__ as g; g.build()" > $O/build_$T.log 2>&1 || { tail -5 $O/build_$T.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "exact or c1_parity_dh" > $O/pytest_$T.log 2>&1; tail -3 $O/pytest_$T.log
run() { n=$1; shift; timeout 600 python bench.py --no-e2e --no-cpu --reps 2 "$@" > $O/bench_${T}_$n.json 2> $O/bench_${T}_$n.err; python - $O/bench_${T}_$n.json $n <<'PY'
import json,sys
try:
    d=json.load(open(sys.argv[1]))
    ph=d['phases_ms_per_step']
    print(sys.argv[2], 'val %.2f G'%(d['value']/1e9), 'ms %.3f'%d['ms_per_step'], 'pmd %.3f'%ph['push_move_deposit'], 'fill %.3f'%ph.get('fill',0), 'sortmove %.3f'%ph.get('sort_move',0), 'frac %.3f'%d['roofline']['frac'], 'hops %.3f'%d['walk']['hops_per_particle_last_step'])
except Exception as e: print(sys.argv[2], 'FAILED', e)
PY
}
run c2_aux1 --config c2
for v in aux2 aux1s3 aux2s3 noaux noauxs3; do OPP_LIB=variants/libopp_$v.so run c2_$v --config c2; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 4 -c 1 -o $O/prof_${T}_aux1 python bench.py --config c2 --steps 2 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-full $?
OPP_LIB=variants/libopp_aux2.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_push_move_deposit_tiled -s 4 -c 1 -o $O/prof_${T}_aux2 python bench.py --config c2 --steps 2 --warmup 3 --reps 1 --no-e2e --no-cpu > /dev/null 2>&1; echo ncu-full $?
ls $O/*.ncu-rep | tail -3
