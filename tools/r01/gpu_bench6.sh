set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python bench.py > $OUT/bench6.json 2> $OUT/bench6.err; echo "bench rc=$?"
tail -1 $OUT/bench6.json | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('value', d['value'], 'link', d['link_roofline']['frac'], 'k1', d['roofline']['frac'])
for k in ('slowdown','slowdown_unpaced','slowdown_graphs'):
    x=d[k]; print(k, x.get('slowdown_pct'), x.get('d2h_gbs'), x.get('iter_ms_no_ckpt'), x.get('error'))"
tail -3 $OUT/bench6.err
