#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
o=gpurun_out/gate_probe2.txt; : > $o
for m in hostwait pageable; do
  for wm in warm warmcold; do
    timeout -s KILL 15 tools/exp/gate_probe $m dev $wm >> $o 2>&1; echo "rc=$? ($m dev $wm)" >> $o
    CUDA_MODULE_LOADING=EAGER timeout -s KILL 15 tools/exp/gate_probe $m dev $wm >> $o 2>&1; echo "rc=$? ($m dev $wm EAGER)" >> $o
  done
done
cat $o
