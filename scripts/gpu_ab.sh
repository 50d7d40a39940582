# A/B of libopp variants: scripts/gpu_ab.sh "<bench args>" name1 name2 ...  (variants/libopp_<name>.so; "cur" = in-tree build)
ARGS="$1"; shift
cp paper_conf_icpp_lantra0m24_b200/libopp.so variants/libopp_cur.so
for rep in 1 2; do
for v in "$@"; do
  cp variants/libopp_$v.so paper_conf_icpp_lantra0m24_b200/libopp.so
  timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu $ARGS 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']
print('$v', round(d['value']/1e9,2), {k: round(x,3) for k,x in p.items()}, 'frac', round(d['roofline']['frac'],3))" || echo "$v failed"
done; done
cp variants/libopp_cur.so paper_conf_icpp_lantra0m24_b200/libopp.so
