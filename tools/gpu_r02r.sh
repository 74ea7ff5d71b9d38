#!/usr/bin/env bash
# round-end style validation on v7: the whole -m gpu suite as the driver runs it, smoke, the default
# C3 bench line (v7 traffic, corrected bidirectional probe) and the C2 line
set -u
mkdir -p gpurun_out
o=gpurun_out/r02r.log; : > $o
timeout -s KILL 3000 python -m pytest tests/ -x -q -m gpu -p no:cacheprovider >> $o 2>&1; echo "pytest-gpu rc=$?" >> $o
timeout -s KILL 120 python -c "import __graft_entry__ as g; g.smoke()" >> $o 2>&1; echo "smoke rc=$?" >> $o
timeout -s KILL 1500 python bench.py > gpurun_out/r02r_bench_c3.json 2> gpurun_out/r02r_bench_c3.err; echo "bench c3 rc=$?" >> $o
timeout -s KILL 900 python bench.py --config c2 > gpurun_out/r02r_bench_c2.json 2> gpurun_out/r02r_bench_c2.err; echo "bench c2 rc=$?" >> $o
tail -6 $o
