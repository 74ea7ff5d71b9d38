"""CPU oracle for the PCcheck snapshot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
``paper_conf_asplos_strati0k25_b200`` never imports it, and nothing here imports the
product.  The arithmetic lives in ``pcc_oracle.c`` (plain, single-threaded C, one byte
at a time); this module only marshals numpy buffers through ctypes.

Each function names the oracle step it runs (O1..O7 of DESIGN.md §3, after SURVEY.md
§8(c)) and the PAPER.md passage it follows.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "pcc_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

ENOENT, ECORRUPT, ELAYOUT, EIO = 1, 2, 3, 4
NONE_ITER = (1 << 64) - 1


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain C, -O2).  Building the checker is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-Wall", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        u8p, u32p, u64p = C.POINTER(C.c_uint8), C.POINTER(C.c_uint32), C.POINTER(C.c_uint64)
        _lib.orc_crc32c.restype = C.c_uint32
        _lib.orc_crc32c.argtypes = [C.c_void_p, C.c_uint64]
        _lib.orc_crc32c_extend.restype = C.c_uint32
        _lib.orc_crc32c_extend.argtypes = [C.c_uint32, C.c_void_p, C.c_uint64]
        _lib.orc_layout.argtypes = [C.c_uint32, u64p, C.c_uint32, C.c_uint64, u64p, u64p, u64p]
        _lib.orc_slice.argtypes = [C.c_uint64, C.c_uint32, C.c_uint32, u64p, u64p]
        _lib.orc_pack.argtypes = [C.c_uint32, C.POINTER(C.c_void_p), u64p, u64p, C.c_uint64, C.c_uint64,
                                  C.c_uint64, C.c_void_p]
        _lib.orc_chunk_crcs.argtypes = [C.c_void_p, C.c_uint64, C.c_uint64, u32p]
        _lib.orc_layout_crc.restype = C.c_uint32
        _lib.orc_layout_crc.argtypes = [C.c_uint32, u64p, u32p, C.c_uint32, C.c_uint64]
        for f in ("orc_header_bytes",):
            getattr(_lib, f).restype = C.c_uint64
            getattr(_lib, f).argtypes = [C.c_uint64]
        _lib.orc_slot_stride.restype = C.c_uint64
        _lib.orc_slot_stride.argtypes = [C.c_uint64, C.c_uint64]
        _lib.orc_slot_offset.restype = C.c_uint64
        _lib.orc_slot_offset.argtypes = [C.c_uint32, C.c_uint64, C.c_uint64]
        _lib.orc_slot_header.argtypes = [C.c_void_p, C.c_uint32, C.c_uint64, C.c_uint64, C.c_uint64, C.c_uint32,
                                         C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32,
                                         C.c_uint32, C.c_uint32, C.c_uint32, u32p]
        _lib.orc_ptr_record.argtypes = [C.c_void_p, C.c_uint32, C.c_uint64, C.c_uint64, C.c_uint64, C.c_uint32,
                                        C.c_uint32, C.c_uint64, C.c_uint32]
        _lib.orc_latest.argtypes = [C.c_char_p, u64p, u64p, u64p]
        _lib.orc_restore.argtypes = [C.c_uint32, C.POINTER(C.c_char_p), C.c_uint32, C.c_uint32, u64p, u32p,
                                     C.c_uint32, C.c_uint64, C.c_uint64, C.c_int, C.POINTER(C.c_void_p), u64p,
                                     u32p, C.c_uint32, u32p]
        _lib.orc_write_checkpoint.argtypes = [C.c_char_p, C.c_uint32, C.POINTER(C.c_void_p), u64p, u32p,
                                              C.c_uint32, C.c_uint64, C.c_uint32, C.c_uint32, C.c_uint32,
                                              C.c_uint32, C.c_uint64, C.c_uint64, C.c_uint64, C.c_uint64, C.c_int]
    return _lib


def _u64(a):
    a = np.ascontiguousarray(np.asarray(a, dtype=np.uint64))
    return a, a.ctypes.data_as(C.POINTER(C.c_uint64))


def _u32(a):
    a = np.ascontiguousarray(np.asarray(a, dtype=np.uint32))
    return a, a.ctypes.data_as(C.POINTER(C.c_uint32))


def _bufs(srcs):
    arrs = [np.ascontiguousarray(np.frombuffer(memoryview(s).cast("B"), dtype=np.uint8)) if not isinstance(s, np.ndarray)
            else np.ascontiguousarray(s).view(np.uint8).reshape(-1) for s in srcs]
    ptrs = (C.c_void_p * max(1, len(arrs)))(*[a.ctypes.data for a in arrs])
    return arrs, ptrs


def crc32c(data) -> int:
    """O3: CRC-32C (reflected 0x82F63B78, init/xorout 0xFFFFFFFF), byte at a time."""
    b = np.frombuffer(bytes(data), dtype=np.uint8) if not isinstance(data, np.ndarray) else np.ascontiguousarray(data).view(np.uint8)
    return int(lib().orc_crc32c(b.ctypes.data, b.nbytes))


def crc32c_extend(crc, data) -> int:
    """O3/O4 resumed: CRC32C(A || data) given crc = CRC32C(A) (crc = 0 for an empty A),
    byte at a time — the slice digest of a multi-GB image in one pass, chunk by chunk."""
    b = np.ascontiguousarray(data).view(np.uint8)
    return int(lib().orc_crc32c_extend(crc, b.ctypes.data, b.nbytes))


def layout(nbytes, align=256, chunk_bytes=4 << 20):
    """O1: image offsets, end and chunk count C (R1-R3; PAPER L127/L281 'contiguous')."""
    nb, nbp = _u64(nbytes)
    off = np.zeros(max(1, len(nb)), dtype=np.uint64)
    end, cnt = C.c_uint64(), C.c_uint64()
    lib().orc_layout(len(nb), nbp, align, chunk_bytes, off.ctypes.data_as(C.POINTER(C.c_uint64)),
                     C.byref(end), C.byref(cnt))
    return off[: len(nb)], int(end.value), int(cnt.value)


def rank_slice(n_chunks, rank, world):
    """Rank r owns chunks [floor(rC/W), floor((r+1)C/W)) (§8(e))."""
    a, b = C.c_uint64(), C.c_uint64()
    lib().orc_slice(n_chunks, rank, world, C.byref(a), C.byref(b))
    return int(a.value), int(b.value)


def pack(srcs, align=256, chunk_bytes=4 << 20, first_chunk=0, count=None):
    """O2: the packed image bytes of chunks [first_chunk, first_chunk+count)."""
    arrs, ptrs = _bufs(srcs)
    nbytes = [a.nbytes for a in arrs]
    off, end, n_chunks = layout(nbytes, align, chunk_bytes)
    if count is None:
        count = n_chunks - first_chunk
    nb, nbp = _u64(nbytes)
    offa, offp = _u64(off)
    out = np.empty(count * chunk_bytes, dtype=np.uint8)
    lib().orc_pack(len(arrs), ptrs, nbp, offp, chunk_bytes, first_chunk, count, out.ctypes.data)
    return out


def pack_chunks_sparse(all_nbytes, srcs_by_index, align, chunk_bytes, first_chunk, count):
    """O2 for chunks [first_chunk, first_chunk+count) of a large registration when only the
    tensors overlapping those chunks are at hand: the layout (O1) comes from ALL sizes, the
    byte copy from the given tensors (every other tensor must not overlap the range)."""
    off, end, c = layout(all_nbytes, align, chunk_bytes)
    lo, hi = first_chunk * chunk_bytes, (first_chunk + count) * chunk_bytes
    idx = sorted(srcs_by_index)
    for i in range(len(all_nbytes)):
        if int(off[i]) < hi and int(off[i]) + int(all_nbytes[i]) > lo and all_nbytes[i] > 0:
            assert i in srcs_by_index, f"tensor {i} overlaps the range but was not given"
    arrs, ptrs = _bufs([srcs_by_index[i] for i in idx])
    nb, nbp = _u64([all_nbytes[i] for i in idx])
    offa, offp = _u64([off[i] for i in idx])
    out = np.empty(count * chunk_bytes, dtype=np.uint8)
    lib().orc_pack(len(idx), ptrs, nbp, offp, chunk_bytes, first_chunk, count, out.ctypes.data)
    return out


def pack_range(all_nbytes, fetch, align, chunk_bytes, first_chunk, count):
    """O2 for image bytes [lo, hi) = [first_chunk*CB, (first_chunk+count)*CB), written with
    numpy slice copies instead of the C byte loop (which walks every byte of every tensor it
    is handed, far too slow to cover a 16-32 GB image chunk by chunk):

        image[max(off_i, lo) - lo : min(off_i + n_i, hi) - lo]
            = tensor_i[max(lo - off_i, 0) : min(hi - off_i, n_i)]     for every tensor i,

    zero everywhere else (R1, R3; "contiguous").  ``fetch(i, a, b)`` returns
    bytes [a, b) of tensor i as a uint8 array.  Pinned against ``pack`` (the C byte loop) by
    brute force in tests/test_oracle.py."""
    off, end, c = layout(all_nbytes, align, chunk_bytes)
    lo, hi = first_chunk * chunk_bytes, (first_chunk + count) * chunk_bytes
    out = np.zeros(hi - lo, dtype=np.uint8)
    for i, n in enumerate(all_nbytes):
        o = int(off[i])
        a, b = max(o, lo), min(o + int(n), hi)
        if b > a:
            piece = np.asarray(fetch(i, a - o, b - o), dtype=np.uint8).reshape(-1)
            assert piece.nbytes == b - a, f"fetch({i}) returned {piece.nbytes} bytes, wanted {b - a}"
            out[a - lo:b - lo] = piece
    return out


def chunk_crcs(img, chunk_bytes):
    """O3 per chunk: crc[c] = CRC32C(image[c*CB:(c+1)*CB])."""
    img = np.ascontiguousarray(img).view(np.uint8)
    count = img.nbytes // chunk_bytes
    out = np.zeros(max(1, count), dtype=np.uint32)
    lib().orc_chunk_crcs(img.ctypes.data, count, chunk_bytes, out.ctypes.data_as(C.POINTER(C.c_uint32)))
    return out[:count]


def layout_crc(nbytes, dtypes, align, chunk_bytes) -> int:
    nb, nbp = _u64(nbytes)
    dt, dtp = _u32(dtypes)
    return int(lib().orc_layout_crc(len(nb), nbp, dtp, align, chunk_bytes))


def header_bytes(n) -> int:
    return int(lib().orc_header_bytes(n))


def slot_offset(slot, n, chunk_bytes) -> int:
    return int(lib().orc_slot_offset(slot, n, chunk_bytes))


def slot_stride(n, chunk_bytes) -> int:
    return int(lib().orc_slot_stride(n, chunk_bytes))


def slot_header(state, iter, counter, chunk_bytes, rank, world, total_chunks, first_chunk, n, n_tensors, align,
                layout_crc_, digest, slot, crcs) -> bytes:
    """O5: the slot header (Listing 1's Check_meta, L250, extended with the CRC table)."""
    out = np.zeros(header_bytes(n), dtype=np.uint8)
    cr, crp = _u32(list(crcs) if n else [0])
    lib().orc_slot_header(out.ctypes.data, state, iter, counter, chunk_bytes, rank, world, total_chunks, first_chunk,
                          n, n_tensors, align, layout_crc_, digest, slot, crp)
    return out.tobytes()


def ptr_record(world, seq, local_iter, local_counter, local_slot, rank, global_iter, n_slots) -> bytes:
    """O5: one of the two alternating persisted CHECK_ADDR records (L229, L277; R7)."""
    out = np.zeros(4096, dtype=np.uint8)
    lib().orc_ptr_record(out.ctypes.data, world, seq, local_iter, local_counter, local_slot, rank, global_iter,
                         n_slots)
    return out.tobytes()


def latest(path):
    g, l, s = C.c_uint64(), C.c_uint64(), C.c_uint64()
    rc = lib().orc_latest(path.encode(), C.byref(g), C.byref(l), C.byref(s))
    if rc:
        return None
    return int(g.value), int(l.value), int(s.value)


def write_checkpoint(path, srcs, dtypes, align, chunk_bytes, rank, world, n_slots, slot, iter, counter, seq,
                     global_iter=None, write_pointer=True):
    """Writes one COMPLETE checkpoint of rank `rank` into `slot` of `path` (+ pointer record)."""
    arrs, ptrs = _bufs(srcs)
    nb, nbp = _u64([a.nbytes for a in arrs])
    dt, dtp = _u32(dtypes)
    rc = lib().orc_write_checkpoint(path.encode(), len(arrs), ptrs, nbp, dtp, align, chunk_bytes, rank, world,
                                    n_slots, slot, iter, counter, seq, iter if global_iter is None else global_iter,
                                    1 if write_pointer else 0)
    if rc:
        raise OSError(f"orc_write_checkpoint rc={rc}")


def restore(paths, n_slots, nbytes, dtypes, align, chunk_bytes, want_iter=None, fallback=False, bad_cap=4096):
    """O7: verify + scatter (L287 §4.2; R10, R13).  Returns (rc, iter, bad_chunks, tensors)."""
    nb, nbp = _u64(nbytes)
    dt, dtp = _u32(dtypes)
    outs = [np.zeros(int(n), dtype=np.uint8) for n in nbytes]
    ptrs = (C.c_void_p * max(1, len(outs)))(*[o.ctypes.data for o in outs])
    cpaths = (C.c_char_p * len(paths))(*[p.encode() for p in paths])
    it = C.c_uint64(0)
    bad = np.zeros(bad_cap, dtype=np.uint32)
    nbad = C.c_uint32(0)
    rc = lib().orc_restore(len(paths), cpaths, n_slots, len(nb), nbp, dtp, align, chunk_bytes,
                           NONE_ITER if want_iter is None else want_iter, 1 if fallback else 0, ptrs,
                           C.byref(it), bad.ctypes.data_as(C.POINTER(C.c_uint32)), bad_cap, C.byref(nbad))
    return rc, int(it.value), [int(x) for x in bad[: min(nbad.value, bad_cap)]], outs
