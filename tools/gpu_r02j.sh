#!/usr/bin/env bash
# v7 with producer fast path, no per-item division, 2 producer + 2 storer warps: parity + A/B
set -u
mkdir -p gpurun_out
o=gpurun_out/r02j.log; : > $o
timeout -s KILL 600 python -m pytest tests/test_kernels_gpu.py -m gpu -x -q -p no:cacheprovider >> $o 2>&1; echo "kernels rc=$?" >> $o
for cfg in c2 c3; do
  for v in default nocrc p4 p1 v6 default v6; do
    lib=""; impl=v7; [ $v != default ] && [ $v != v6 ] && lib=build/$v/libpccheck.so; [ $v = v6 ] && impl=v6
    PCC_LIB=$lib PCC_KIMPL=$impl timeout -s KILL 300 python tools/k1_bench.py --config $cfg --reps 7 >> $o 2>&1; echo "$cfg $v rc=$?" >> $o
  done
done
timeout -s KILL 600 ncu --set full --import-source on --clock-control none -k regex:k_snap_tma --launch-skip 2 -c 1 -o gpurun_out/r02j_v7_c2 \
  python tools/k1_bench.py --config c2 --reps 3 > gpurun_out/r02j_ncu.log 2>&1; echo "ncu rc=$?" >> $o
cat $o
