set -u
OUT=gpurun_out; mkdir -p $OUT
ISO_KINDS="none,d2h,trickle:0:4:64,trickle:30:4:64,trickle:20:2:32,trickle:30:8:16,trickle:15:2:16" timeout 900 python tools/slowdown_iso.py > $OUT/iso3.jsonl 2>&1
for q in 1 0.5 0.25; do
 for p in 20 30 40; do
  PCC_D2H_GBS=$p PCC_D2H_QUANTUM_MIB=$q ISO_KINDS=none,ckpt timeout 600 python tools/slowdown_iso.py 2>&1 | grep ckpt >> $OUT/iso3.jsonl
 done
done
cat $OUT/iso3.jsonl | cut -c1-250
