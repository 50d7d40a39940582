run() { timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu "$@" 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,2), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items() if k in ('push_move_deposit','fill')})"; }
cp paper_conf_icpp_lantra0m24_b200/libopp.so /tmp/libopp_base.so
cp variants/libopp_s2.so paper_conf_icpp_lantra0m24_b200/libopp.so
for c in 100 86 72 61; do echo "s2 carve $c"; OPP_CARVEOUT=$c run; done
cp variants/libopp_s3.so paper_conf_icpp_lantra0m24_b200/libopp.so
for c in 100 86 79; do echo "s3 carve $c"; OPP_CARVEOUT=$c run; done
cp /tmp/libopp_base.so paper_conf_icpp_lantra0m24_b200/libopp.so
for c in 100 96; do echo "base carve $c"; OPP_CARVEOUT=$c run; done
