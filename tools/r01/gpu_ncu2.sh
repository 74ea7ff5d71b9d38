set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_snapshot -s 2 -c 1 -o $OUT/k1v5_full -f python tools/k1_bench.py --config c2 --cb 16777216 --reps 4 > /dev/null 2>&1; echo "ncu k1 rc=$?"
PCC_LIB=build/va_nocrc/libpccheck.so timeout 600 ncu --set full --clock-control none -k regex:k_snapshot -s 2 -c 1 -o $OUT/k1nocrc_full -f python tools/k1_bench.py --config c2 --cb 16777216 --reps 4 > /dev/null 2>&1; echo "ncu nocrc rc=$?"
