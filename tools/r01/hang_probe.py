"""Runs one runtime scenario with a watchdog that dumps thread states if it hangs."""
import faulthandler, os, sys, threading, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("PCC_TRACE", "1")

def watchdog(sec):
    time.sleep(sec)
    print("=== WATCHDOG: hung; thread states ===", file=sys.stderr, flush=True)
    for t in sorted(os.listdir("/proc/self/task")):
        try:
            comm = open(f"/proc/self/task/{t}/comm").read().strip()
            wchan = open(f"/proc/self/task/{t}/wchan").read().strip()
            st = open(f"/proc/self/task/{t}/stat").read().split()[2]
            print(t, comm, st, wchan, file=sys.stderr)
        except Exception as e:
            print(t, e, file=sys.stderr)
    faulthandler.dump_traceback(all_threads=True)
    os._exit(3)

threading.Thread(target=watchdog, args=(float(sys.argv[2]) if len(sys.argv) > 2 else 60,), daemon=True).start()
import torch
import paper_conf_asplos_strati0k25_b200 as pcc
from synth import config_tensors, make_state, perturb_state
mode = sys.argv[1] if len(sys.argv) > 1 else "pwrite_odirect"
flags = {"mapfile": pcc.MAPFILE, "pwrite_odirect": pcc.ODIRECT | pcc.FSYNC, "pwrite": pcc.ODIRECT}[mode]
specs = config_tensors("c1")
ts = make_state(specs, "cuda", seed=1, it=0)
path = f"/dev/shm/pcc_hang_{os.getpid()}.pcc"
with pcc.PCCheck(path, chunk_bytes=4 << 20, max_inflight=2, flags=flags, staging_bytes=16 << 20) as ck:
    ck.register(ts)
    for it in (10, 20, 30):
        perturb_state(ts, specs, 1, it)
        h = ck.checkpoint(it)
        ck.guard()
        ck.wait(h)
        print("ok", it, ck.info(h)["state_name"], file=sys.stderr, flush=True)
os.unlink(path)
print("DONE", file=sys.stderr)
