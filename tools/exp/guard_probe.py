"""Diagnostic: does the GPU-side U-gate (cuStreamWaitValue32 in pcc_guard) release the training
stream?  One process, C1 state: checkpoint -> guard -> a D2H on the training stream, timed."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch  # noqa: E402
import paper_conf_asplos_strati0k25_b200 as pcc  # noqa: E402
from synth import config_tensors, make_state, perturb_state  # noqa: E402

specs = config_tensors("c1")
ts = make_state(specs, "cuda", seed=1, it=0)
path = f"/dev/shm/pcc_guard_probe_{os.getpid()}.pcc"
side = torch.cuda.Stream() if len(sys.argv) > 1 and sys.argv[1] == "side" else None
with pcc.PCCheck(path, chunk_bytes=4 << 20, max_inflight=2, flags=pcc.MAPFILE) as ck:
    ck.register(ts)
    for it in range(1, 6):
        s = side or torch.cuda.current_stream()
        with torch.cuda.stream(s):
            t0 = time.perf_counter()
            h = ck.checkpoint(it, s)
            ck.guard(s)
            t1 = time.perf_counter()
            perturb_state(ts, specs, seed=1, it=it)
            x = ts[0].cpu()
            t2 = time.perf_counter()
            ck.wait(h)
            t3 = time.perf_counter()
        print(f"it {it}: call+guard {1e3 * (t1 - t0):.2f} ms, stream through the gate {1e3 * (t2 - t1):.2f} ms, "
              f"wait {1e3 * (t3 - t2):.2f} ms, state {ck.info(h)['state_name']}", flush=True)
os.unlink(path)
print("guard probe ok")
