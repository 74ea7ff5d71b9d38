#!/usr/bin/env bash
# D2H copy size A/B in MAPFILE mode (PCC_COALESCE_MIB): bench value and idle snapshot
set -u
for m in 64 256 1024 64 256 1024; do
  PCC_COALESCE_MIB=$m timeout 600 python bench.py --no-slowdown --no-cpu-baseline --steps 20 2>/dev/null | tail -1 | \
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print($m, round(d['value'],2), round(d['link_roofline']['frac'],3), round(d['snapshot_idle']['ms'],2), round(d['e2e']['value'],1), round(d['restore']['gbs'],1))"
done
