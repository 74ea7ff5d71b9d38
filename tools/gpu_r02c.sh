#!/usr/bin/env bash
# round 2: the GPU suite again after the U-gate redesign (each file under its own timeout)
set -u
mkdir -p gpurun_out
o=gpurun_out/r02c_pytest.log; : > $o
timeout -s KILL 120 python tools/exp/guard_probe.py >> $o 2>&1; echo "guard probe rc=$?" >> $o
for f in tests/test_runtime_gpu.py tests/test_kernels_gpu.py tests/test_crash_gpu.py tests/test_dp_gpu.py \
         tests/test_dp_crash_gpu.py tests/test_tuner.py tests/test_fullsize_gpu.py; do
  echo "== $f" >> $o
  timeout -s KILL 2000 python -m pytest $f -m gpu -q -p no:cacheprovider --durations=5 >> $o 2>&1
  echo "rc=$?" >> $o
done
grep -E "^==|passed|failed|rc=|error" $o | tail -40
