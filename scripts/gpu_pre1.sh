python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -5 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2
run() { timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --field 0 "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill','continue')}, d['walk']['hops_per_particle_last_step'])"; }
echo "pre1"; run
echo "pre1 mh"; run --mh
cp variants/libopp_pre0.so paper_conf_icpp_lantra0m24_b200/libopp.so
echo "pre0"; run
cp variants/libopp_pre1.so paper_conf_icpp_lantra0m24_b200/libopp.so
echo "pre1 again"; run
