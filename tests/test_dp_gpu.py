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


def _rank_main(rank, world, tmpdir, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = {}
    try:
        import paper_conf_asplos_strati0k25_b200 as pcc
        torch.cuda.set_device(0)
        specs = config_tensors("c1")
        ts = make_state(specs, "cuda", seed=31, it=0)  # replicated DP state: same seed on every rank

        path = os.path.join(tmpdir, f"r{rank}.pcc")
        saved = {}
        with pcc.PCCheck(path, chunk_bytes=CB, max_inflight=2, flags=pcc.MAPFILE, rank=rank, world=world,
                         **pcc.torch_collectives(dist)) as ck:
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


def test_dp_world2_on_one_gpu(shmdir):
    tmp_path = __import__("pathlib").Path(shmdir)  # MAPFILE needs a DRAM-backed file
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 33500 + os.getpid() % 1000
    procs = [ctx.Process(target=_rank_main, args=(r, 2, str(tmp_path), port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(2))
    for p in procs:
        p.join(60)
    for r in range(2):
        assert "error" not in res[r], res[r].get("error")
    import paper_conf_asplos_strati0k25_b200 as pcc
    assert res[0]["slice"] == (0, 8, 17) and res[1]["slice"] == (8, 9, 17)
    for r in range(2):
        assert (res[r]["g10"], res[r]["g20"], res[r]["g30"]) == (10, 20, 30)
        assert res[r]["restore"] == 30 and res[r]["restore_ok"]
        assert res[r]["corrupt_rc"] == pcc.ECORRUPT
        assert res[r]["fallback"] == 20 and res[r]["fallback_ok"]
    # the oracle, reading both rank files, agrees (with fallback past the corrupted slice)
    specs = config_tensors("c1")
    paths = [str(tmp_path / f"r{r}.pcc") for r in range(2)]
    rc, it, bad, outs = oracle.restore(paths, 3, [s.nbytes for s in specs], [s.code for s in specs], 256, CB,
                                       fallback=True)
    assert rc == 0 and it == 20
