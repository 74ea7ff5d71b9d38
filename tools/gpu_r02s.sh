#!/usr/bin/env bash
# handle-validity test + runtime suite; the f3 sweeps with K1 v7; OPT-1.3B graphs x K1 grid cap
set -u
mkdir -p gpurun_out
o=gpurun_out/r02s.log; : > $o
timeout -s KILL 900 python -m pytest tests/test_runtime_gpu.py -m gpu -q -p no:cacheprovider >> $o 2>&1; echo "runtime rc=$?" >> $o
timeout -s KILL 3000 python tools/sweeps.py > gpurun_out/r02s_sweeps.jsonl 2> gpurun_out/r02s_sweeps.err; echo "sweeps rc=$?" >> $o
timeout -s KILL 2400 bash tools/gpu_graph_packctas_v7.sh >> $o 2>&1; echo "packctas rc=$?" >> $o
tail -12 $o
