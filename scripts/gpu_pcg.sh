python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 300 python scripts/field_probe.py 2>&1 | grep -v "^dbg\|^bps" | tail -12
echo "classic CG"; OPP_CG_PIPE=0 timeout 300 python scripts/field_probe.py 2>&1 | grep "precond 1 tol 1e-10\|warm"
run() { timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill','continue','sort_move','field')}, d.get('field',{}).get('cg_iterations_last'))"; }
echo "bench field on"; run
echo "bench field off"; run --field 0
cp variants/libopp_minb4.so paper_conf_icpp_lantra0m24_b200/libopp.so
echo "minb4 field off"; run --field 0
cp variants/libopp_base.so paper_conf_icpp_lantra0m24_b200/libopp.so
