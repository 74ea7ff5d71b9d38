"""Parity at BASELINE.json's full sizes, in the bench's launch configuration (DRAM-file target,
full-slice HBM ring): EVERY chunk of the slot byte for byte, the WHOLE header CRC table and the
slice digest, each against the oracle (SURVEY §8(c) "GPU vs oracle").

The expected image comes from ``oracle.pack_range`` (O2 as numpy slice copies, pinned against the
C byte loop in test_oracle.py) over the state's bytes copied to the host by torch — never from
the CUDA path.  Expected CRCs are ``oracle.crc32c`` (byte-at-a-time Sarwate) of those chunks on a
thread pool; the expected digest is ONE sequential ``oracle.crc32c_extend`` pass over the whole
slice (O4's definition, no combine).  K2's restore is then checked as an identity on top."""
import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np
import pytest

import oracle
from synth import config_tensors, make_state, perturb_state

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(1500)]
torch = pytest.importorskip("torch")
MiB = 1 << 20


@pytest.fixture(scope="module")
def pcc():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_asplos_strati0k25_b200 as p
    return p


def _tmp(name):
    d = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
    return os.path.join(d, f"pcc_full_{name}_{os.getpid()}.pcc")


def _bytes_of(t):
    return (t.reshape(-1) if t.dim() else t.reshape(1)).view(torch.uint8)


def oracle_check_slot(path, specs, ts, slot, n, first, cb, align=256):
    """Every chunk, the CRC table and the digest of `slot` in the rank file `path` vs the
    oracle.  Returns (chunks compared, the oracle digest)."""
    nbytes = [s.nbytes for s in specs]
    flat = [_bytes_of(t) for t in ts]

    def fetch(i, a, b):  # tensor i's bytes [a, b), device -> host by torch (independent of K1)
        return flat[i][a:b].cpu().numpy()

    H = oracle.header_bytes(n)
    base = oracle.slot_offset(slot, n, cb)
    mm = np.memmap(path, dtype=np.uint8, mode="r")
    hdr = np.array(mm[base:base + H])
    crc_tab = hdr[96:96 + 4 * n].view("<u4").tolist()
    digest_hdr = int(hdr[72:76].view("<u4")[0])
    assert int(hdr[8:12].view("<u4")[0]) == 2, "slot header not COMPLETE"
    workers = max(2, min(16, (os.cpu_count() or 4) - 2))
    crc_pool, dig_pool = ThreadPoolExecutor(workers), ThreadPoolExecutor(1)  # ctypes drops the GIL
    digest = [0]

    def extend(img):  # runs strictly in submission order (one worker): a single pass over the slice
        digest[0] = oracle.crc32c_extend(digest[0], img)

    crc_futs, dig_futs, bad = [], [], []
    try:
        for j in range(n):
            exp = oracle.pack_range(nbytes, fetch, align, cb, first + j, 1)
            got = mm[base + H + j * cb: base + H + (j + 1) * cb]
            if not np.array_equal(got, exp):
                bad.append(first + j)
            crc_futs.append(crc_pool.submit(oracle.crc32c, exp))
            dig_futs.append(dig_pool.submit(extend, exp))
            if j >= 24:  # bound the chunks held in host memory
                dig_futs[j - 24].result()
        crcs = [f.result() for f in crc_futs]
        for f in dig_futs:
            f.result()
    finally:
        crc_pool.shutdown(wait=True)
        dig_pool.shutdown(wait=True)
        del mm
    assert not bad, f"{len(bad)} of {n} chunks differ from the oracle image, first {bad[:8]}"
    mism = [first + j for j in range(n) if crcs[j] != crc_tab[j]]
    assert not mism, f"header CRC32C differs from the oracle for chunks {mism[:8]}"
    assert digest[0] == digest_hdr, f"slice digest {digest_hdr:08x} != oracle {digest[0]:08x}"
    return n, digest[0]


@pytest.mark.parametrize("cfg,emulate,cb", [("c2", 0, 16 * MiB), ("c3", 0, 64 * MiB), ("c4", 8, 64 * MiB)])
def test_full_size_every_chunk_vs_oracle(pcc, cfg, emulate, cb):
    """c2 at the bench's 16 MiB chunks (the whole 1.1 GB image); c3 = OPT-1.3B + Adam (15.79 GB,
    236 chunks); c4 = BLOOM-7b1 mixed-precision Adam as rank 0 of 8 (the 12.3 GB slice of a
    98.97 GB registration) — every chunk, the CRC table and the digest vs the oracle."""
    specs = config_tensors(cfg)
    ts = make_state(specs, "cuda", seed=9, it=1)
    path = _tmp(cfg)
    before = None
    flags = pcc.MAPFILE | (pcc.NOCOMM if emulate else 0)
    try:
        with pcc.PCCheck(path, chunk_bytes=cb, max_inflight=1, flags=flags, world=emulate or 1) as ck:
            ck.register(ts)
            h = ck.checkpoint(10)
            ck.wait(h)
            ck.commit()  # global commit (with PCC_NOCOMM the rank reduces over itself)
            inf = ck.info(h, with_crc=True)
            geo = ck.geometry()
            n = geo["count"]
            assert (geo["first"], n) == oracle.rank_slice(geo["n_chunks"], 0, emulate or 1)  # c4: (0, 184) of 1475
            cnt, dig = oracle_check_slot(path, specs, ts, inf["slot"], n, geo["first"], cb)
            assert cnt == n and inf["digest"] == dig and len(inf["crc"]) == n
            # restore (K2 verify + scatter) is an identity on top: the tensors inside the slice
            offs, _, _ = oracle.layout([sp.nbytes for sp in specs], 256, cb)
            hi = (geo["first"] + n) * cb
            inside = [i for i in range(len(specs)) if int(offs[i]) + specs[i].nbytes <= hi]
            inside = inside[:: max(1, len(inside) // 16)]
            before = [ts[i].clone() for i in inside]
            perturb_state(ts, specs, seed=9, it=2)
            it, bad = ck.restore()
            assert it == 10 and bad == []
            assert all(torch.equal(_bytes_of(a), _bytes_of(ts[i])) for a, i in zip(before, inside))
    finally:
        ts = before = None
        torch.cuda.empty_cache()
        if os.path.exists(path):
            os.unlink(path)


def test_c5_restore_faults_full_size(pcc):
    """BASELINE configs[4] on one GPU: OPT-2.7B state (31.8 GB).  The first checkpoint is
    checked against the oracle in full (every chunk, CRC table, digest); then k = 8 seeded faults
    in the newest checkpoint -> ECORRUPT naming exactly those chunks; PCC_FALLBACK -> the older
    checkpoint, bit-exact (restore is an identity, checked on the device at full size)."""
    CB = 64 * MiB
    specs = config_tensors("c5")
    ts = make_state(specs, "cuda", seed=5, it=10)
    path = _tmp("c5")
    s10 = None
    try:
        with pcc.PCCheck(path, chunk_bytes=CB, max_inflight=1, flags=pcc.MAPFILE) as ck:
            ck.register(ts)
            h10 = ck.checkpoint(10)
            ck.wait(h10)
            n = ck.geometry()["count"]
            oracle_check_slot(path, specs, ts, ck.info(h10)["slot"], n, 0, CB)
            s10 = [t.clone() for t in ts]
            perturb_state(ts, specs, seed=5, it=20)
            h20 = ck.checkpoint(20)
            ck.wait(h20)
            slot = ck.info(h20)["slot"]
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
                assert torch.equal(_bytes_of(a), _bytes_of(b))
    finally:
        ts = s10 = None
        torch.cuda.empty_cache()
        if os.path.exists(path):
            os.unlink(path)
