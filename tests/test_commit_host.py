"""The library's commit engine (pccheck_host.h) on CPU: Listing 1 against the oracle's
sequential model, on-file bytes against the oracle's format, crash points, resume, and the
data-parallel rule under torch.distributed gloo with world_size 2."""
import os
import random

import numpy as np
import pytest

import oracle
from oracle.manager_model import ListingOne

pcc = pytest.importorskip("paper_conf_asplos_strati0k25_b200")

CB = 4096
SIZES = [5000, 17, 12000, 0, 40000, 3]


def _state(seed):
    rng = np.random.default_rng(seed)
    return [rng.integers(0, 256, n, dtype=np.uint8) for n in SIZES]


def _geom():
    off, end, c = oracle.layout(SIZES, 256, CB)
    return c, oracle.layout_crc(SIZES, [0] * len(SIZES), 256, CB)


def _engine(path, N=2, rank=0, world=1):
    c, lcrc = _geom()
    return pcc.HostEngine(path, CB, N, rank, world, c, len(SIZES), 256, lcrc)


def _write_data(e, path, slot, state, rank=0, world=1):
    """What the persist threads do (here from the oracle's packed image of this rank's slice)."""
    c, _ = _geom()
    first, n = oracle.rank_slice(c, rank, world)
    img = oracle.pack(state, 256, CB, first_chunk=first, count=n)
    with open(path, "r+b") as f:
        f.seek(e.data_offset(slot))
        f.write(img.tobytes())
    return [int(x) for x in oracle.chunk_crcs(img, CB)], oracle.crc32c(img)


def test_listing1_matches_sequential_model(tmp_path):
    rng = random.Random(3)
    for trial in range(20):
        path = str(tmp_path / f"t{trial}.pcc")
        N = rng.choice([1, 2, 3])
        e = _engine(path, N)
        m = ListingOne(N)
        inflight, it = [], 0
        for step in range(60):
            if inflight and (rng.random() < 0.5 or len(inflight) == N + (1 if m.CHECK_ADDR is None else 0)):
                k = rng.randrange(len(inflight))
                (counter, slot, mck) = inflight.pop(k)
                st = e.complete(counter, [0] * _geom()[0], 0)
                mst = m.persisted(mck)
                assert pcc.STATE_NAMES[st] == mst
            else:
                it += 10
                got = e.begin(it)
                mck = m.begin(it)
                assert (got is None) == (mck is None)
                if got is None:
                    continue
                assert got == (mck.counter, mck.data_location)
                inflight.append((got[0], got[1], mck))
            assert e.free_slots() == len(m.free_space)
            if m.CHECK_ADDR is not None:
                assert pcc.latest(path) == (m.CHECK_ADDR.iter, m.CHECK_ADDR.iter)
        e.close()


def test_file_bytes_match_oracle_and_oracle_restores(tmp_path):
    path = str(tmp_path / "f.pcc")
    e = _engine(path, 2)
    c, lcrc = _geom()
    for it in (10, 20, 30):
        counter, slot = e.begin(it)
        e.filling(counter)
        s = _state(it)
        crcs, dig = _write_data(e, path, slot, s)
        assert e.complete(counter, crcs, dig) == pcc.ST_LOCAL_COMMIT
        exp = oracle.slot_header(2, it, counter, CB, 0, 1, c, 0, c, len(SIZES), 256, lcrc, dig, slot, crcs)
        with open(path, "rb") as f:
            f.seek(oracle.slot_offset(slot, c, CB))
            assert f.read(len(exp)) == exp
            f.seek(4096 * ((counter + 1) % 2))
            assert f.read(4096) == oracle.ptr_record(1, counter + 1, it, counter, slot, 0, it, 3)
        rc, rit, bad, outs = oracle.restore([path], 3, SIZES, [0] * len(SIZES), 256, CB)
        assert rc == 0 and rit == it and all(np.array_equal(o, x) for o, x in zip(outs, s))
    e.close()


@pytest.mark.parametrize("crash_at", ["after_begin", "after_filling", "mid_data", "before_complete"])
def test_crash_points_keep_last_commit(tmp_path, crash_at):
    """Stop the protocol at each point of FORMAT.md's commit order: restore must give the
    previous committed iter, bit-exact (R18, R19)."""
    path = str(tmp_path / "c.pcc")
    e = _engine(path, 1)  # N=1: iter 20 reuses... a free slot, iter 30 would reuse 10's slot
    for it in (10, 20):
        counter, slot = e.begin(it)
        e.filling(counter)
        crcs, dig = _write_data(e, path, slot, _state(it))
        e.complete(counter, crcs, dig)
    counter, slot = e.begin(30)  # reuses iter 10's slot
    s30 = _state(30)
    if crash_at != "after_begin":
        e.filling(counter)
    if crash_at in ("mid_data", "before_complete"):
        c, _ = _geom()
        img = oracle.pack(s30, 256, CB)
        with open(path, "r+b") as f:
            f.seek(e.data_offset(slot))
            f.write(img.tobytes()[: (len(img) // 2 if crash_at == "mid_data" else len(img))])
    e.close()  # the process dies here
    rc, it, bad, outs = oracle.restore([path], 2, SIZES, [0] * len(SIZES), 256, CB, fallback=True)
    assert rc == 0 and it == 20
    assert all(np.array_equal(o, x) for o, x in zip(outs, _state(20)))
    # the library resumes on the same file: 20's slot is not reusable, counters continue
    e2 = _engine(path, 1)
    assert e2.local_latest() == 20
    counter, slot = e2.begin(40)
    crcs, dig = _write_data(e2, path, slot, _state(40))
    assert e2.complete(counter, crcs, dig) == pcc.ST_LOCAL_COMMIT
    rc, it, bad, outs = oracle.restore([path], 2, SIZES, [0] * len(SIZES), 256, CB)
    assert rc == 0 and it == 40
    e2.close()


def test_torn_pointer_record_falls_back(tmp_path):
    path = str(tmp_path / "p.pcc")
    e = _engine(path, 2)
    for it in (10, 20):
        counter, slot = e.begin(it)
        crcs, dig = _write_data(e, path, slot, _state(it))
        e.complete(counter, crcs, dig)
    e.close()
    with open(path, "r+b") as f:  # seq 2 (iter 20) lives at offset 0: tear it
        f.seek(100)
        f.write(b"\xde\xad")
    assert pcc.latest(path) == (10, 10)
    rc, it, bad, outs = oracle.restore([path], 3, SIZES, [0] * len(SIZES), 256, CB)
    assert rc == 0 and it == 10


# ------------------------------------------------------------------ DP under gloo
def _dp_worker(rank, world, tmpdir, seed, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        path = os.path.join(tmpdir, f"r{rank}.pcc")
        N = 2
        e = _engine(path, N, rank, world)
        rng = random.Random(seed * 100 + rank)  # ranks persist in different orders
        inflight, it, checks = [], 0, 0
        committed = {}
        for step in range(40):
            # collective backpressure: everybody begins together or nobody does
            need = torch.tensor([0 if e.free_slots() else 1])
            dist.all_reduce(need, op=dist.ReduceOp.MAX)
            if need.item() == 0:
                it += 10
                counter, slot = e.begin(it)
                e.filling(counter)
                inflight.append((counter, slot, it))
            # persist some in random order
            rng.shuffle(inflight)
            keep = []
            for (counter, slot, i) in inflight:
                if rng.random() < 0.5:
                    crcs, dig = _write_data(e, path, slot, _state(i), rank, world)
                    e.complete(counter, crcs, dig)
                    committed[i] = True
                else:
                    keep.append((counter, slot, i))
            inflight = keep
            L = e.local_latest()
            g = torch.tensor([-1 if L is None else L])
            dist.all_reduce(g, op=dist.ReduceOp.MIN)
            if g.item() >= 0:
                e.apply_global(g.item())
                held = e.held()
                assert g.item() in held, (rank, g.item(), held)  # every rank keeps g (R8)
                checks += 1
        for (counter, slot, i) in inflight:
            crcs, dig = _write_data(e, path, slot, _state(i), rank, world)
            e.complete(counter, crcs, dig)
        L = e.local_latest()
        g = torch.tensor([L])
        dist.all_reduce(g, op=dist.ReduceOp.MIN)
        e.apply_global(g.item())
        e.close()
        dist.barrier()
        q.put((rank, checks, int(g.item())))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("seed", [0, 1])
def test_dp_commit_gloo_world2(tmp_path, seed):
    import torch.multiprocessing as mp
    port = 29500 + (os.getpid() + seed) % 2000
    os.environ["MASTER_PORT"] = str(port)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_dp_worker, args=(r, 2, str(tmp_path), seed, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
        assert p.exitcode == 0
    res = sorted(q.get() for _ in range(2))
    g = res[0][2]
    assert res[0][2] == res[1][2] and res[0][1] > 0
    paths = [str(tmp_path / f"r{r}.pcc") for r in range(2)]
    rc, it, bad, outs = oracle.restore(paths, 3, SIZES, [0] * len(SIZES), 256, CB)
    assert rc == 0 and it == g
    assert all(np.array_equal(o, x) for o, x in zip(outs, _state(g)))


# ----------------------------------------------- restore agreement under gloo (pcc_restore's W>1 logic)
def _verify_with_oracle(path, e, slot):
    """The test's stand-in for K2 on this rank's slice: recompute every chunk CRC32C with the
    oracle and compare with the slot header's table."""
    import struct as _s
    first, n, _ = e.geometry()
    with open(path, "rb") as f:
        f.seek(oracle.slot_offset(slot, n, CB))
        hdr = f.read(oracle.header_bytes(n))
        f.seek(e.data_offset(slot))
        data = np.frombuffer(f.read(n * CB), dtype=np.uint8)
    if data.nbytes < n * CB:
        return False
    table = list(_s.unpack_from(f"<{n}I", hdr, 96)) if n else []
    return [int(x) for x in oracle.chunk_crcs(data, CB)] == table


def _agree_worker(rank, world, tmpdir, scenario, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        path = os.path.join(tmpdir, f"r{rank}.pcc")
        e = _engine(path, 2, rank, world)
        for it in (10, 20, 30):
            counter, slot = e.begin(it)
            e.filling(counter)
            if not (scenario == "rank1_missing_30" and rank == 1 and it == 30):  # else: 30 never durable here
                crcs, dig = _write_data(e, path, slot, _state(it), rank, world)
                e.complete(counter, crcs, dig)
            L = torch.tensor([e.local_latest()])
            dist.all_reduce(L, op=dist.ReduceOp.MIN)
            e.apply_global(int(L.item()))
        if scenario == "corrupt_rank1_latest" and rank == 1:
            held = e.held()
            g = e.global_iter()
            with open(path, "r+b") as f:
                f.seek(e.data_offset(held[g]) + 123)
                b = f.read(1)
                f.seek(e.data_offset(held[g]) + 123)
                f.write(bytes([b[0] ^ 0x80]))

        def reduce(v, is_max):
            t = torch.tensor([v], dtype=torch.int64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX if is_max else dist.ReduceOp.MIN)
            return int(t.item())

        try:
            got = e.restore_plan(reduce, lambda it, slot: _verify_with_oracle(path, e, slot), fallback=True)
        except pcc.PCCError as ex:
            got = -ex.code
        e.close()
        q.put((rank, got))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("scenario", ["clean", "rank1_missing_30", "corrupt_rank1_latest"])
def test_restore_agreement_gloo_world2(tmp_path, scenario):
    import torch.multiprocessing as mp
    os.environ["MASTER_PORT"] = str(31500 + (os.getpid() + len(scenario)) % 2000)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_agree_worker, args=(r, 2, str(tmp_path), scenario, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
        assert p.exitcode == 0
    res = dict(q.get() for _ in range(2))
    assert res[0] == res[1], res  # every rank restores the same iter
    paths = [str(tmp_path / f"r{r}.pcc") for r in range(2)]
    rc, it, bad, outs = oracle.restore(paths, 3, SIZES, [0] * len(SIZES), 256, CB, fallback=True)
    assert rc == 0 and res[0] == it  # ... the one the oracle picks from the same files
    expect = {"clean": 30, "rank1_missing_30": 20, "corrupt_rank1_latest": 20}[scenario]
    assert it == expect
