python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2
run() { timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --field 0 "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill','continue')}, d['walk']['hops_per_particle_last_step'])"; }
echo "full"; run
echo "dbg4"; OPP_PMD_DEBUG=4 run
for ov in 0.0625 0.25 0.5; do echo "ov $ov"; run --ov $ov; done
echo "dep0"; run --deposit 0
