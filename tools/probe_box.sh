#!/usr/bin/env bash
# Box probe, SURVEY §7 step 0. Writes gpurun_out/probe/*.txt
set -u
OUT=${1:-gpurun_out/probe}
mkdir -p "$OUT"
{
  nvidia-smi; nvidia-smi topo -m
  nvidia-smi --query-gpu=index,pci.bus_id,pcie.link.gen.max,pcie.link.gen.current,pcie.link.width.max,pcie.link.width.current --format=csv
} > "$OUT/nvidia.txt" 2>&1
{ lscpu; nproc; cat /proc/meminfo | head -5; numactl -H 2>/dev/null; ls /sys/devices/system/node/ ; cat /sys/bus/pci/devices/*/numa_node 2>/dev/null | sort | uniq -c; } > "$OUT/host.txt" 2>&1
{ df -h; lsblk; mount | grep -E ' / | /dev/shm | /tmp ' ; cat /sys/kernel/mm/transparent_hugepage/enabled; uname -a; ulimit -l; } > "$OUT/storage.txt" 2>&1
python - > "$OUT/odirect.txt" 2>&1 <<'EOF'
import os, mmap, time
for d in ["/dev/shm", "/tmp", "/root", os.environ.get("GRAFT_REPO_ROOT", ".")]:
    p = os.path.join(d, "pcc_odirect_probe.bin")
    try:
        fd = os.open(p, os.O_RDWR | os.O_CREAT | os.O_DIRECT, 0o600)
        buf = mmap.mmap(-1, 64 << 20)
        buf.write(b"\x5a" * (64 << 20))
        t = time.perf_counter()
        for i in range(8):
            os.pwrite(fd, buf, i * (64 << 20))
        os.fsync(fd)
        dt = time.perf_counter() - t
        print(d, "O_DIRECT ok", f"{8*64/1024/dt:.2f} GiB/s")
        os.close(fd); os.unlink(p)
    except Exception as e:
        print(d, "O_DIRECT failed", repr(e))
EOF
timeout 300 ./tools/probe 0 > "$OUT/probe_gpu0.jsonl" 2>&1
ncu --version > "$OUT/ncu.txt" 2>&1
ncu --query-metrics 2>/dev/null | grep -iE 'pcie|sysmem|dram__bytes' >> "$OUT/ncu.txt" 2>&1
echo done
