"""Isolates the per-checkpoint training cost seen in tools/slowdown_diag.py: the VGG-16 loop
with, after the step of every 10th iteration, ONE of: nothing; a 1.1 GB D2H copy-engine
transfer on a side stream; a 1.1 GB HBM->HBM SM copy on a side stream; both; the library's
checkpoint.  Prints the extra ms of each iteration position vs the plain loop."""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch
    import torchvision
    import paper_conf_asplos_strati0k25_b200 as pcc
    torch.manual_seed(0)
    model = torchvision.models.vgg16(weights=None).cuda()
    opt = torch.optim.SGD(model.parameters(), lr=1e-3, momentum=0.9)
    x = torch.randn(32, 3, 224, 224, device="cuda")
    y = torch.randint(0, 1000, (32,), device="cuda")
    lossf = torch.nn.CrossEntropyLoss()
    ts = torch.cuda.current_stream()
    side = torch.cuda.Stream()
    nb = 1106860352
    dsrc = torch.empty(nb, dtype=torch.uint8, device="cuda")
    ddst = torch.empty(nb, dtype=torch.uint8, device="cuda")
    hdst = torch.empty(nb, dtype=torch.uint8).pin_memory()

    def fwd_bwd():
        opt.zero_grad(set_to_none=True)
        lossf(model(x), y).backward()

    for _ in range(3):
        fwd_bwd()
        opt.step()
    use_graph = os.environ.get("ISO_GRAPH") == "1"
    if use_graph:  # two graphs so the U-gate could sit between them
        s0 = torch.cuda.Stream()
        s0.wait_stream(ts)
        with torch.cuda.stream(s0):
            for _ in range(3):
                fwd_bwd()
                opt.step()
        ts.wait_stream(s0)
        g1, g2 = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
        opt.zero_grad(set_to_none=True)
        with torch.cuda.graph(g1):
            lossf(model(x), y).backward()
        with torch.cuda.graph(g2):
            opt.step()

        def step():
            g1.replay()
            g2.replay()
    else:
        def step():
            fwd_bwd()
            opt.step()
    state = []
    for p in model.parameters():
        state += [p.data, opt.state[p]["momentum_buffer"]]
    ck = pcc.PCCheck(os.path.join("/dev/shm", f"iso_{os.getpid()}.pcc"), chunk_bytes=64 << 20, max_inflight=2,
                     flags=pcc.MAPFILE, d2h_gbs=float(os.environ.get("PCC_D2H_GBS", "0")),
                     d2h_quantum=int(float(os.environ.get("PCC_D2H_QUANTUM_MIB", "0")) * (1 << 20)))
    ck.register(state)
    it = [0]
    import ctypes as C
    trk = C.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "exp", "libtrickle.so"))
    trk.trickle.argtypes = [C.c_void_p, C.c_void_p, C.c_uint64, C.c_double, C.c_uint32, C.c_uint32, C.c_void_p]
    for k in os.environ.get("ISO_KINDS", "").split(","):  # standalone rate of each trickle config
        if k.startswith("trickle"):
            _, g, n, kb = k.split(":")
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(side)
            trk.trickle(C.c_void_p(dsrc.data_ptr()), C.c_void_p(hdst.data_ptr()), C.c_uint64(nb), C.c_double(float(g)),
                        int(n), int(kb) << 10, C.c_void_p(side.cuda_stream))
            b.record(side)
            b.synchronize()
            print(json.dumps({"trickle_alone": k, "gbs": nb / (a.elapsed_time(b) * 1e-3) / 1e9}), flush=True)

    def act(kind):
        if kind == "none":
            return
        if kind == "sleep5":  # is the host ahead of the GPU? (if so this costs nothing)
            time.sleep(0.005)
            return
        side.wait_stream(ts)
        if kind.startswith("trickle"):  # trickle:<GB/s>:<ctas>:<block KiB>
            _, g, n, kb = kind.split(":")
            rc = trk.trickle(C.c_void_p(dsrc.data_ptr()), C.c_void_p(hdst.data_ptr()), C.c_uint64(nb),
                             C.c_double(float(g)), int(n), int(kb) << 10, C.c_void_p(side.cuda_stream))
            assert rc == 0, rc
            return
        with torch.cuda.stream(side):
            if kind in ("d2h", "both"):
                hdst.copy_(dsrc, non_blocking=True)
            if kind in ("d2d_sm", "both"):
                torch.add(dsrc, 0, out=ddst)
            if kind == "d2d_ce":
                ddst.copy_(dsrc, non_blocking=True)
        if kind == "ckpt":
            it[0] += 1
            ck.checkpoint(it[0], ts)

    def loop(kind, n=60, every=10):
        per = []
        e0 = torch.cuda.Event(enable_timing=True)
        e0.record(ts)
        last = e0
        for i in range(1, n + 1):
            step()
            if i % every == 0:
                act(kind)
            ev = torch.cuda.Event(enable_timing=True)
            ev.record(ts)
            per.append((last, ev))
            last = ev
        torch.cuda.synchronize()
        ck.drain()
        return [a.elapsed_time(b) for a, b in per]

    loop("none", 20)
    kinds = os.environ.get("ISO_KINDS", "none,sleep5,d2h,d2d_sm,d2d_ce,both,ckpt").split(",")
    pos = {k: [[] for _ in range(10)] for k in kinds}
    for r in range(3):
        for k in kinds:
            for i, v in enumerate(loop(k)):
                pos[k][(i + 1) % 10].append(v)
    base = [statistics.mean(v) for v in pos["none"]]
    for k in kinds:
        m = [statistics.mean(v) for v in pos[k]]
        print(json.dumps({"kind": k, "graph": use_graph, "pace": os.environ.get("PCC_D2H_GBS"),
                          "quantum_mib": os.environ.get("PCC_D2H_QUANTUM_MIB"), "iter_ms": round(statistics.mean(m), 3),
                          "extra_ms_by_pos": [round(a - b, 3) for a, b in zip(m, base)]}), flush=True)
    ck.close()
    os.unlink(os.path.join("/dev/shm", f"iso_{os.getpid()}.pcc"))


if __name__ == "__main__":
    main()
