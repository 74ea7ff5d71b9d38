"""Parity at BASELINE.json's full sizes, in the bench's launch configuration (64 MiB chunks,
DRAM-file target, full-slice HBM ring): sampled chunks against the oracle, and restore as an
identity at any size (C5 with injected faults)."""
import os

import numpy as np
import pytest

import oracle
from synth import config_tensors, make_state, perturb_state, host_bytes

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(900)]
torch = pytest.importorskip("torch")
CB = 64 << 20


@pytest.fixture(scope="module")
def pcc():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_asplos_strati0k25_b200 as p
    return p


def _tmp(name):
    d = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    return os.path.join(d, f"pcc_full_{name}_{os.getpid()}.pcc")


def _sampled_parity(path, specs, ts, slot, n, first, sample):
    nbytes = [s.nbytes for s in specs]
    off, end, C = oracle.layout(nbytes, 256, CB)
    for j in sample:
        g = first + j
        lo, hi = g * CB, (g + 1) * CB
        need = {i: host_bytes(t) for i, t in enumerate(ts)
                if nbytes[i] and int(off[i]) < hi and int(off[i]) + nbytes[i] > lo}
        exp = oracle.pack_chunks_sparse(nbytes, need, 256, CB, g, 1)
        with open(path, "rb") as f:
            f.seek(oracle.slot_offset(slot, n, CB) + oracle.header_bytes(n) + j * CB)
            got = np.frombuffer(f.read(CB), dtype=np.uint8)
            f.seek(oracle.slot_offset(slot, n, CB) + 96 + 4 * j)
            crc = int(np.frombuffer(f.read(4), dtype=np.uint32)[0])
        assert np.array_equal(got, exp), f"chunk {g} differs"
        assert crc == oracle.crc32c(exp), f"chunk {g} CRC"


@pytest.mark.parametrize("cfg,emulate", [("c3", 0), ("c4", 8)])
def test_full_size_sampled_chunks(pcc, cfg, emulate):
    specs = config_tensors(cfg)
    ts = make_state(specs, "cuda", seed=9, it=1)
    path = _tmp(cfg)
    flags = pcc.MAPFILE | (pcc.NOCOMM if emulate else 0)
    try:
        with pcc.PCCheck(path, chunk_bytes=CB, max_inflight=1, flags=flags, world=emulate or 1) as ck:
            ck.register(ts)
            h = ck.checkpoint(10)
            ck.wait(h)
            ck.commit()  # global commit (with PCC_NOCOMM the rank reduces over itself)
            inf = ck.info(h)
            geo = ck.geometry()
            n = geo["count"]
            rng = np.random.default_rng(0)
            sample = sorted({0, n - 1, n // 2, *rng.integers(0, n, 3).tolist()})
            _sampled_parity(path, specs, ts, inf["slot"], n, geo["first"], sample)
            # digest consistency: the header digest equals the CRC32C of the file's slice bytes
            # recomputed from the per-chunk CRCs the header lists is not independent; instead
            # re-verify the whole slice with K2 via restore (identity at any size)
            # with PCC_NOCOMM only this rank's slice is restored: compare the tensors inside it
            offs, _, _ = oracle.layout([sp.nbytes for sp in specs], 256, CB)
            hi = (geo["first"] + n) * CB
            inside = [i for i in range(len(specs)) if int(offs[i]) + specs[i].nbytes <= hi][:8]
            before = [ts[i].clone() for i in inside]
            perturb_state(ts, specs, seed=9, it=2)
            it, bad = ck.restore()
            assert it == 10 and bad == []
            assert all(torch.equal(a.view(-1).view(torch.uint8) if a.dim() else a.reshape(1).view(torch.uint8),
                                   b.view(-1).view(torch.uint8) if b.dim() else b.reshape(1).view(torch.uint8))
                       for a, b in zip(before, [ts[i] for i in inside]))
    finally:
        ts = None
        torch.cuda.empty_cache()
        if os.path.exists(path):
            os.unlink(path)


def test_c5_restore_faults_full_size(pcc):
    """BASELINE configs[4] on one GPU: OPT-2.7B state (31.8 GB), k = 8 seeded faults in the
    newest checkpoint -> ECORRUPT naming exactly those chunks; PCC_FALLBACK -> the older
    checkpoint, bit-exact (restore is an identity, checked on the device at full size)."""
    specs = config_tensors("c5")
    ts = make_state(specs, "cuda", seed=5, it=10)
    path = _tmp("c5")
    try:
        with pcc.PCCheck(path, chunk_bytes=CB, max_inflight=1, flags=pcc.MAPFILE) as ck:
            ck.register(ts)
            ck.wait(ck.checkpoint(10))
            s10 = [t.clone() for t in ts]
            perturb_state(ts, specs, seed=5, it=20)
            h20 = ck.checkpoint(20)
            ck.wait(h20)
            slot = ck.info(h20)["slot"]
            n = ck.geometry()["count"]
            rng = np.random.default_rng(8)
            chunks = sorted(rng.choice(n, 8, replace=False).tolist())
            kinds = ["bitflip", "burst32", "half_stale", "zero_tail", "bitflip", "burst32", "half_stale", "zero_tail"]
            other = 1 - slot
            with open(path, "r+b") as f:
                for j, kind in zip(chunks, kinds):
                    base = oracle.slot_offset(slot, n, CB) + oracle.header_bytes(n) + j * CB
                    f.seek(base)
                    cur = f.read(CB)
                    if kind == "bitflip":
                        new, at = bytes([cur[4097] ^ 0x01]), 4097
                    elif kind == "burst32":
                        new, at = bytes(b ^ 0xFF for b in cur[100:104]), 100
                    elif kind == "half_stale":
                        f.seek(oracle.slot_offset(other, n, CB) + oracle.header_bytes(n) + j * CB + CB // 2)
                        new, at = f.read(CB // 2), CB // 2
                    else:
                        new, at = bytes(4096), CB - 4096
                    if new == cur[at:at + len(new)]:  # the injector must change bytes
                        new = bytes(b ^ 0x5A for b in new)
                    f.seek(base + at)
                    f.write(new)
            perturb_state(ts, specs, seed=5, it=99)
            with pytest.raises(pcc.PCCError) as ei:
                ck.restore()
            assert ei.value.code == pcc.ECORRUPT and sorted(ei.value.bad_chunks) == chunks
            it, bad = ck.restore(fallback=True)
            assert it == 10
            for a, b in zip(ts, s10):
                assert torch.equal(a.reshape(-1).view(torch.uint8), b.reshape(-1).view(torch.uint8))
    finally:
        ts = s10 = None
        torch.cuda.empty_cache()
        if os.path.exists(path):
            os.unlink(path)
