set -u
OUT=gpurun_out; mkdir -p $OUT
for q in 0 256 512 1024 2048; do
  timeout 600 python bench.py --no-slowdown --no-cpu-baseline --d2h-quantum-kib $q > $OUT/bq_$q.json 2>$OUT/bq_$q.err
  python -c "
import json; d=json.loads(open('$OUT/bq_$q.json').read().strip().splitlines()[-1])
print('q=$q', 'value %.2f'%d['value'], 'link %.3f'%d['link_roofline']['frac'], 'e2e %.2f'%d['e2e']['value'], 'lat %.1f'%d['checkpoint_latency_ms_p50'], 'k1 %.3f'%d['roofline']['launch_ms'])"
done
timeout 600 python bench.py --no-slowdown --no-cpu-baseline --config c3 --inflight 4 --d2h-quantum-kib 512 > $OUT/bq_c3.json 2>$OUT/bq_c3.err
python -c "
import json; d=json.loads(open('$OUT/bq_c3.json').read().strip().splitlines()[-1])
print('c3 q=512', 'value %.2f'%d['value'], 'link %.3f'%d['link_roofline']['frac'], 'e2e %.2f'%d['e2e']['value'], 'lat %.1f'%d['checkpoint_latency_ms_p50'])"
