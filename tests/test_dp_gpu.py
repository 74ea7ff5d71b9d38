"""The data-parallel path of the library on ONE GPU: two rank processes share cuda:0 and use
gloo (through pcc_config's allreduce/allgather callbacks) instead of NCCL.  This runs the real
W = 2 code: 1/W slicing, the commit allreduce(MIN), collective backpressure, the restore
agreement (MAX / MIN / MAX), the allgather fan-out of verified chunks and K2 on the other
rank's chunks — checked against the oracle restoring both rank files."""
import os

import numpy as np
import pytest

import oracle
from synth import config_tensors, make_state, perturb_state, host_bytes

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(300)]
torch = pytest.importorskip("torch")
CB = 4 << 20


def _rank_main(rank, world, tmpdir, port, q, transport="gloo"):
    """transport="gloo": every rank on cuda:0, the library's collectives through gloo callbacks;
    "nccl": rank r on cuda:r with the library's OWN NCCL communicator (gloo only carries the
    128-byte unique id and the test's barriers)."""
    import faulthandler
    import torch.distributed as dist
    faulthandler.dump_traceback_later(200, exit=True)  # a hung rank shows where, then exits
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = {}
    try:
        import paper_conf_asplos_strati0k25_b200 as pcc
        dev = rank if transport == "nccl" else 0
        torch.cuda.set_device(dev)
        if transport == "nccl":
            obj = [pcc.nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0)
            coll = {"nccl_unique_id": obj[0], "device": dev}
        else:
            coll = pcc.torch_collectives(dist)
        specs = config_tensors("c1")
        ts = make_state(specs, "cuda", seed=31, it=0)  # replicated DP state: same seed on every rank

        path = os.path.join(tmpdir, f"r{rank}.pcc")
        saved = {}
        with pcc.PCCheck(path, chunk_bytes=CB, max_inflight=2, flags=pcc.MAPFILE, rank=rank, world=world,
                         **coll) as ck:
            ck.register(ts)
            geo = ck.geometry()
            out["slice"] = (geo["first"], geo["count"], geo["n_chunks"])
            for it in (10, 20, 30):
                perturb_state(ts, specs, 31, it)
                h = ck.checkpoint(it)
                ck.guard()
                ck.wait(h)
                out[f"g{it}"] = ck.commit()
                saved[it] = [host_bytes(t).copy() for t in ts]
            # restore fan-out: own slice from the file + the other rank's slice over the collective
            perturb_state(ts, specs, 31, 99)
            it, bad = ck.restore()
            out["restore"] = it
            out["restore_ok"] = all(np.array_equal(host_bytes(t), s) for t, s in zip(ts, saved[30]))
            rs = ck.restore_stats()  # pcc_restore_stats at W = 2: the fan-out is timed too
            out["restore_stats_ok"] = (rs["attempts"] == 1 and rs["bytes"] == geo["count"] * CB and rs["fanout_ms"] > 0
                                       and rs["k2_ms"] > 0 and rs["total_ms"] >= rs["fanout_ms"])
            # rank 1's newest slice is corrupted -> every rank must reject 30 and agree on 20
            dist.barrier()
            if rank == 1:
                n = geo["count"]
                with open(path, "r+b") as f:
                    for s in range(3):
                        f.seek(oracle.slot_offset(s, n, CB) + 16)
                        if int(np.frombuffer(f.read(8), dtype=np.uint64)[0]) == 30:
                            off = oracle.slot_offset(s, n, CB) + oracle.header_bytes(n) + 1234
                            f.seek(off)
                            b = f.read(1)
                            f.seek(off)
                            f.write(bytes([b[0] ^ 0x40]))
            dist.barrier()
            try:
                ck.restore()
                out["corrupt_rc"] = 0
            except pcc.PCCError as e:
                out["corrupt_rc"] = e.code
            perturb_state(ts, specs, 31, 98)
            it, bad = ck.restore(fallback=True)
            out["fallback"] = it
            out["fallback_ok"] = all(np.array_equal(host_bytes(t), s) for t, s in zip(ts, saved[20]))
    except Exception as e:  # noqa: BLE001
        out["error"] = repr(e)
    finally:
        q.put((rank, out))
        dist.destroy_process_group()


@pytest.fixture
def shmdir(tmp_path):
    import shutil
    import tempfile
    d = tempfile.mkdtemp(dir="/dev/shm") if os.path.isdir("/dev/shm") else str(tmp_path)
    yield d
    shutil.rmtree(d, ignore_errors=True)


@pytest.mark.parametrize("transport", ["gloo", "nccl"])
def test_dp_world2(shmdir, transport):
    """gloo: two ranks share cuda:0 (runs on any GPU box).  nccl: two ranks on two GPUs with the
    library's own NCCL communicator (ncclAllReduce MIN/MAX for commit and agreement, ncclAllGather
    for the restore fan-out over NVLink); skipped when fewer than 2 GPUs are visible."""
    tmp_path = __import__("pathlib").Path(shmdir)  # MAPFILE needs a DRAM-backed file
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    if transport == "nccl" and torch.cuda.device_count() < 2:
        pytest.skip("the native NCCL path needs 2 GPUs")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 33500 + os.getpid() % 1000 + (7 if transport == "nccl" else 0)
    procs = [ctx.Process(target=_rank_main, args=(r, 2, str(tmp_path), port, q, transport), daemon=True)
             for r in range(2)]
    for p in procs:
        p.start()
    try:
        res = dict(q.get(timeout=230) for _ in range(2))
        for p in procs:
            p.join(60)
    finally:  # never leave a hung rank behind (pytest would wait for it at exit)
        for p in procs:
            if p.is_alive():
                p.kill()
    for r in range(2):
        assert "error" not in res[r], res[r].get("error")
    import paper_conf_asplos_strati0k25_b200 as pcc
    assert res[0]["slice"] == (0, 8, 17) and res[1]["slice"] == (8, 9, 17)
    for r in range(2):
        assert (res[r]["g10"], res[r]["g20"], res[r]["g30"]) == (10, 20, 30)
        assert res[r]["restore"] == 30 and res[r]["restore_ok"] and res[r]["restore_stats_ok"]
        assert res[r]["corrupt_rc"] == pcc.ECORRUPT
        assert res[r]["fallback"] == 20 and res[r]["fallback_ok"]
    # the oracle, reading both rank files, agrees (with fallback past the corrupted slice)
    specs = config_tensors("c1")
    paths = [str(tmp_path / f"r{r}.pcc") for r in range(2)]
    rc, it, bad, outs = oracle.restore(paths, 3, [s.nbytes for s in specs], [s.code for s in specs], 256, CB,
                                       fallback=True)
    assert rc == 0 and it == 20


def _c5_rank(rank, world, tmpdir, port, q):
    """C5 (OPT-2.7B, 31.8 GB) at W = 2 on one GPU: checkpoint 10, then 20 with faults injected
    into BOTH ranks' slices; the restore must name exactly this rank's bad chunks (ECORRUPT), and
    PCC_FALLBACK must agree on 10 on both ranks and restore it bit for bit (own slice from the
    file, the other rank's through the allgather fan-out + K2)."""
    import faulthandler
    import torch.distributed as dist
    faulthandler.dump_traceback_later(1050, exit=True)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = {}
    cb = 64 << 20
    try:
        import paper_conf_asplos_strati0k25_b200 as pcc
        torch.cuda.set_device(0)
        specs = config_tensors("c5")
        ts = make_state(specs, "cuda", seed=55, it=10)
        path = os.path.join(tmpdir, f"c5_r{rank}.pcc")
        with pcc.PCCheck(path, chunk_bytes=cb, max_inflight=1, flags=pcc.MAPFILE, rank=rank, world=world,
                         **pcc.torch_collectives(dist)) as ck:
            ck.register(ts)
            h10 = ck.checkpoint(10)
            ck.wait(h10)
            assert ck.commit() == 10
            crc10 = ck.info(h10, with_crc=True)["crc"]
            # sampled tensors across the WHOLE image (both ranks' slices) kept on the device
            keep = {i: ts[i].clone() for i in list(range(0, len(ts), 37)) + [len(ts) - 1]}
            perturb_state(ts, specs, 55, 20)
            h = ck.checkpoint(20)
            ck.wait(h)
            assert ck.commit() == 20
            geo = ck.geometry()
            n, first, slot = geo["count"], geo["first"], ck.info(h)["slot"]
            rng = np.random.default_rng(100 + rank)
            local = sorted(rng.choice(n, 4, replace=False).tolist())
            with open(path, "r+b") as f:
                for k, j in enumerate(local):
                    at = oracle.slot_offset(slot, n, cb) + oracle.header_bytes(n) + j * cb + 4096 * (k + 1) + 7
                    f.seek(at)
                    b = f.read(4)
                    f.seek(at)
                    f.write(bytes(x ^ 0xA5 for x in b))  # a 32-bit burst
            out["bad_expected"] = [first + j for j in local]
            dist.barrier()
            perturb_state(ts, specs, 55, 99)
            try:
                ck.restore()
                out["rc"] = 0
            except pcc.PCCError as e:
                out["rc"] = e.code
                out["bad"] = sorted(e.bad_chunks)
            it, bad = ck.restore(fallback=True)
            out["fallback"] = it
            same = all(torch.equal(a.reshape(-1).view(torch.uint8) if a.dim() else a.reshape(1).view(torch.uint8),
                                   ts[i].reshape(-1).view(torch.uint8) if ts[i].dim() else ts[i].reshape(1).view(torch.uint8))
                       for i, a in keep.items())
            # and this rank's whole slice: re-checkpointing the restored state gives iter 10's table
            h30 = ck.checkpoint(30)
            ck.wait(h30)
            out["identity"] = bool(same and ck.info(h30, with_crc=True)["crc"] == crc10)
            dist.barrier()
    except Exception as e:  # noqa: BLE001
        import traceback
        out["error"] = traceback.format_exc()[-2000:]
    finally:
        q.put((rank, out))
        dist.destroy_process_group()


@pytest.mark.timeout(1200)
def test_dp_c5_faults_world2_on_one_gpu(shmdir):
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import torch.multiprocessing as mp
    import paper_conf_asplos_strati0k25_b200 as pcc
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 34700 + os.getpid() % 1000
    procs = [ctx.Process(target=_c5_rank, args=(r, 2, shmdir, port, q), daemon=True) for r in range(2)]
    for p in procs:
        p.start()
    try:
        res = dict(q.get(timeout=1100) for _ in range(2))
        for p in procs:
            p.join(60)
    finally:
        for p in procs:
            if p.is_alive():
                p.kill()
    for r in range(2):
        assert "error" not in res[r], res[r].get("error")
        assert res[r]["rc"] == pcc.ECORRUPT and res[r]["bad"] == res[r]["bad_expected"], res[r]
        assert res[r]["fallback"] == 10 and res[r]["identity"], res[r]
