#!/usr/bin/env bash
# round 2 (session 2): TMA-staged K1/K2 (v7) parity + same-box A/B against the register path (v6)
set -u
mkdir -p gpurun_out
o=gpurun_out/r02g.log; : > $o
timeout -s KILL 600 python -m pytest tests/test_kernels_gpu.py -m gpu -x -q -p no:cacheprovider >> $o 2>&1; echo "kernels rc=$?" >> $o
timeout -s KILL 120 python -c "import __graft_entry__ as g; g.smoke()" >> $o 2>&1; echo "smoke rc=$?" >> $o
for cfg in c2 c3; do
  for impl in v7 v6 v7 v6; do
    PCC_KIMPL=$impl timeout -s KILL 300 python tools/k1_bench.py --config $cfg --reps 7 >> $o 2>&1; echo "$cfg $impl pack rc=$?" >> $o
  done
  for impl in v7 v6; do
    PCC_KIMPL=$impl timeout -s KILL 300 python tools/k1_bench.py --config $cfg --reps 7 --unpack >> $o 2>&1; echo "$cfg $impl unpack rc=$?" >> $o
  done
done
timeout -s KILL 900 python -m pytest tests/test_runtime_gpu.py -m gpu -x -q -p no:cacheprovider >> $o 2>&1; echo "runtime rc=$?" >> $o
tail -60 $o
