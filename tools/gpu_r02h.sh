#!/usr/bin/env bash
# v7 bottleneck hunt: variant builds (store lag, no-CRC pipeline ceiling, consumer warps) + one ncu --set full of v7 on C2
set -u
mkdir -p gpurun_out
o=gpurun_out/r02h.log; : > $o
for v in default lag6 nocrc nocrc_lag6 w12 w4; do
  lib=""; [ $v != default ] && lib=build/$v/libpccheck.so
  PCC_LIB=$lib timeout -s KILL 300 python tools/k1_bench.py --config c2 --reps 7 >> $o 2>&1; echo "c2 $v rc=$?" >> $o
done
PCC_KIMPL=v6 timeout -s KILL 300 python tools/k1_bench.py --config c2 --reps 7 >> $o 2>&1; echo "c2 v6 rc=$?" >> $o
timeout -s KILL 600 ncu --set full --import-source on --clock-control none -k regex:k_snap_tma -c 1 -o gpurun_out/r02h_v7_c2 \
  python tools/k1_bench.py --config c2 --reps 2 > gpurun_out/r02h_ncu.log 2>&1; echo "ncu rc=$?" >> $o
cat $o
