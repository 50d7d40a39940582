run() { timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu --field 0 "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill','continue','sort_move')})"; }
echo "base"; run
echo "direct"; run --direct
cp variants/libopp_gout.so paper_conf_icpp_lantra0m24_b200/libopp.so
echo "gout (STG out)"; run
echo "gout minb1"; OPP_MINB=1 run
cp variants/libopp_base.so paper_conf_icpp_lantra0m24_b200/libopp.so
echo "base tile_group 4"; OPP_TILE_GROUP=4 run
echo "base tile_group 64"; OPP_TILE_GROUP=64 run
echo "base prefetch"; OPP_PREFETCH=1 run
