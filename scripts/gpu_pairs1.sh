python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
OPP_PAIRS=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -4
run() { timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --field 0 "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill','continue')}, d['walk']['hops_per_particle_last_step'])"; }
echo "base"; run
cp variants/libopp_p4.so paper_conf_icpp_lantra0m24_b200/libopp.so
echo "pairs minb4"; OPP_PAIRS=1 run
echo "pairs minb4 mh"; OPP_PAIRS=1 run --mh
echo "pairs minb4 dep0"; OPP_PAIRS=1 run --deposit 0
cp variants/libopp_p3.so paper_conf_icpp_lantra0m24_b200/libopp.so
echo "pairs minb3"; OPP_PAIRS=1 run
