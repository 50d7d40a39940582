# A/B of an environment knob on one library: scripts/gpu_env_ab.sh VAR "<bench args>" v1 v2 ...
VAR=$1; ARGS=$2; shift 2
for rep in 1 2; do for v in "$@"; do
  env $VAR=$v timeout 300 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu $ARGS 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']
print('$VAR=$v', round(d['value']/1e9,2), {k: round(x,3) for k,x in p.items()}, 'frac', round(d['roofline']['frac'],3))" || echo "$v failed"
done; done
