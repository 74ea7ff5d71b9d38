"""paper_conf_asplos_strati0k25_b200 — B200-native PCcheck snapshot path (Python binding).

A thin ctypes binding over ``libpccheck.so`` (include/pccheck.h, pccheck_kernels.h,
pccheck_host.h).  Argument marshalling only: every step of the checkpoint path (pack,
CRC32C, copy, persist, commit, verify, scatter) runs in the native library.  torch is
used for device pointers and streams only.  There is no fallback: if the library is
missing, importing this package raises.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PCC_LIB") or os.path.join(_HERE, "libpccheck.so")  # PCC_LIB: dev A/B builds

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: run `make` (or __graft_entry__.build()) first; "
                      "the PCcheck path has no non-native fallback")

_lib = C.CDLL(LIB_PATH)

# ---------------------------------------------------------------------- constants
ABI_VERSION = 2
NONE = LATEST = (1 << 64) - 1
OK, EINVAL, ENOMEM, EBUSY, EAGAIN, EIO, ECUDA, ENCCL, EORDER, ECORRUPT, ELAYOUT, ENOENT, ETIMEDOUT, ESTATE = range(14)
ODIRECT, FSYNC, ZEROCOPY, NULLSINK, MAPFILE, NOCOMM, SHARDED, D2H_UPFRONT = 1, 2, 4, 8, 16, 32, 64, 128
FALLBACK = 1
(ST_QUEUED, ST_PACKING, ST_PACKED, ST_PERSISTED, ST_LOCAL_COMMIT, ST_GLOBAL_COMMIT, ST_OBSOLETE,
 ST_FAILED) = range(8)
STATE_NAMES = ["QUEUED", "PACKING", "PACKED", "PERSISTED", "LOCAL_COMMIT", "GLOBAL_COMMIT", "OBSOLETE", "FAILED"]
DTYPE = {"u8": 0, "f32": 1, "bf16": 2, "f16": 3, "f64": 4, "i64": 5, "i32": 6}


class Config(C.Structure):
    _fields_ = [("abi_version", C.c_uint32), ("path", C.c_char_p), ("chunk_bytes", C.c_uint64),
                ("max_inflight", C.c_uint32), ("staging_bytes", C.c_uint64), ("ring_bytes", C.c_uint64),
                ("writer_threads", C.c_uint32), ("flags", C.c_uint32), ("device", C.c_int32), ("rank", C.c_int32),
                ("world", C.c_int32), ("nccl_unique_id", C.c_void_p), ("align", C.c_uint32),
                ("pack_ctas", C.c_uint32), ("allreduce", C.c_void_p), ("allgather", C.c_void_p),
                ("coll_ctx", C.c_void_p), ("d2h_mbps", C.c_uint32), ("d2h_quantum", C.c_uint32)]


ALLREDUCE_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.POINTER(C.c_int64), C.c_uint32, C.c_int)
ALLGATHER_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint64)


class Tensor(C.Structure):
    _fields_ = [("dev_ptr", C.c_void_p), ("nbytes", C.c_uint64), ("dtype", C.c_uint32), ("name", C.c_char_p)]


class RestoreInfo(C.Structure):  # pcc_restore_info
    _fields_ = [("bytes", C.c_uint64), ("attempts", C.c_uint32), ("total_ms", C.c_float), ("read_ms", C.c_float),
                ("h2d_ms", C.c_float), ("k2_ms", C.c_float), ("finalize_ms", C.c_float), ("fanout_ms", C.c_float)]


class Info(C.Structure):
    _fields_ = [("iter", C.c_uint64), ("counter", C.c_uint64), ("slot", C.c_uint32), ("state", C.c_uint32),
                ("digest", C.c_uint32), ("n_chunks", C.c_uint32), ("t_call_us", C.c_double),
                ("t_packed_us", C.c_double), ("t_landed_us", C.c_double), ("t_persisted_us", C.c_double),
                ("t_committed_us", C.c_double), ("pack_ms", C.c_float), ("finalize_ms", C.c_float),
                ("k1_busy_ms", C.c_float), ("snapshot_ms", C.c_float)]


class HostConfig(C.Structure):
    _fields_ = [("path", C.c_char_p), ("chunk_bytes", C.c_uint64), ("max_inflight", C.c_uint32),
                ("rank", C.c_uint32), ("world", C.c_uint32), ("total_chunks", C.c_uint32),
                ("n_tensors", C.c_uint32), ("align", C.c_uint32), ("layout_crc", C.c_uint32),
                ("fsync", C.c_uint32)]


_P, _u32p, _u64p = C.c_void_p, C.POINTER(C.c_uint32), C.POINTER(C.c_uint64)
_SIGS = {
    "pcc_open": (C.c_int, [C.POINTER(Config), C.POINTER(C.c_void_p)]),
    "pcc_register": (C.c_int, [_P, C.POINTER(Tensor), C.c_uint32]),
    "pcc_checkpoint": (C.c_int, [_P, C.c_uint64, _P, _u64p]),
    "pcc_guard": (C.c_int, [_P, _P]),
    "pcc_poll": (C.c_int, [_P, C.c_uint64, C.POINTER(C.c_int)]),
    "pcc_wait": (C.c_int, [_P, C.c_uint64, C.c_int64]),
    "pcc_drain": (C.c_int, [_P, C.c_int64]),
    "pcc_commit": (C.c_int, [_P, _u64p]),
    "pcc_latest": (C.c_int, [C.c_char_p, _u64p, _u64p]),
    "pcc_restore": (C.c_int, [_P, C.c_uint64, C.c_uint32, _u64p, _u32p, C.c_uint32, _u32p]),
    "pcc_info": (C.c_int, [_P, C.c_uint64, C.POINTER(Info), _u32p, C.c_uint32]),
    "pcc_geometry": (C.c_int, [_P, _u64p, _u64p, _u64p, _u64p]),
    "pcc_kernel_launches": (C.c_uint64, [_P]),
    "pcc_close": (C.c_int, [_P]),
    "pcc_nccl_unique_id": (C.c_int, [_P]),
    "pcc_struct_size": (C.c_uint64, [C.c_int]),
    "pcc_restore_stats": (C.c_int, [_P, _P]),
    "pcc_strerror": (C.c_char_p, [C.c_int]),
    "pcc_last_error": (C.c_char_p, []),
    "pcc_last_errno": (C.c_int, []),
    "pcc_k_pack": (C.c_int, [C.POINTER(Tensor), C.c_uint32, C.c_uint32, C.c_uint64, C.c_uint64, C.c_uint64, _P,
                             _P, _P, _P]),
    "pcc_k_unpack": (C.c_int, [C.POINTER(Tensor), C.c_uint32, C.c_uint32, C.c_uint64, C.c_uint64, C.c_uint64,
                               _P, _P, _P, _P, _P, _P]),
    "pcc_k_layout": (C.c_int, [C.POINTER(Tensor), C.c_uint32, C.c_uint32, C.c_uint64, _u64p, _u64p, _u64p]),
    "pcc_k_nccl_selftest": (C.c_int, [C.c_int, C.POINTER(C.c_int64), C.c_uint32, C.POINTER(C.c_int64),
                                      C.POINTER(C.c_int64), C.POINTER(C.c_uint32)]),
    "pcc_host_open": (C.c_int, [C.POINTER(HostConfig), C.POINTER(C.c_void_p)]),
    "pcc_host_begin": (C.c_int, [_P, C.c_uint64, _u64p, _u32p]),
    "pcc_host_filling": (C.c_int, [_P, C.c_uint64]),
    "pcc_host_complete": (C.c_int, [_P, C.c_uint64, _u32p, C.c_uint32, C.POINTER(C.c_int)]),
    "pcc_host_fail": (C.c_int, [_P, C.c_uint64]),
    "pcc_host_state": (C.c_int, [_P, C.c_uint64, C.POINTER(C.c_int)]),
    "pcc_host_local_latest": (C.c_uint64, [_P]),
    "pcc_host_global": (C.c_uint64, [_P]),
    "pcc_host_apply_global": (C.c_int, [_P, C.c_uint64]),
    "pcc_host_free_slots": (C.c_uint32, [_P]),
    "pcc_host_geometry": (C.c_int, [_P, _u32p, _u32p, _u32p]),
    "pcc_host_data_offset": (C.c_uint64, [_P, C.c_uint32]),
    "pcc_host_held": (C.c_uint32, [_P, _u64p, _u32p, C.c_uint32]),
    "pcc_host_restore_plan": (C.c_int, [_P, C.c_uint64, C.c_uint32, _P, _P, _P, _u64p]),
    "pcc_host_close": (C.c_int, [_P]),
}
REDUCE_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.POINTER(C.c_int64), C.c_int)
VERIFY_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_uint64, C.c_uint32)
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args


class PCCError(RuntimeError):
    def __init__(self, code, where=""):
        self.code = -code if code < 0 else code
        detail = (_lib.pcc_last_error() or b"").decode(errors="replace")
        super().__init__(f"{where}: {_lib.pcc_strerror(code).decode()} ({detail})")


def _check(rc, where):
    if rc != 0:
        raise PCCError(rc, where)
    return rc


def exported_symbols():
    return list(_SIGS)


# ------------------------------------------------------------------ tensor marshalling
def _dtype_code(t):
    import torch
    return {torch.float32: 1, torch.bfloat16: 2, torch.float16: 3, torch.float64: 4, torch.int64: 5,
            torch.int32: 6, torch.uint8: 0}.get(t.dtype, 0)


def tensor_table(tensors, names=None):
    """pcc_tensor[] for torch tensors (contiguous) or (ptr, nbytes, dtype_code) tuples."""
    arr = (Tensor * max(1, len(tensors)))()
    keep = []
    for i, t in enumerate(tensors):
        if isinstance(t, tuple):
            ptr, nbytes, code = t
        else:
            if not t.is_contiguous():
                raise ValueError(f"tensor {i} is not contiguous")
            ptr, nbytes, code = t.data_ptr(), t.numel() * t.element_size(), _dtype_code(t)
        nm = (names[i] if names else "").encode()
        keep.append(nm)
        arr[i] = Tensor(C.c_void_p(ptr), nbytes, code, nm)
    return arr, keep


def _stream_ptr(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return stream if isinstance(stream, int) else stream.cuda_stream


# ------------------------------------------------------------------------ the manager
class PCCheck:
    """One pcc_ctx: N-in-flight concurrent checkpoints of registered tensors (PAPER §3-4)."""

    def __init__(self, path=None, chunk_bytes=64 << 20, max_inflight=2, staging_bytes=0, ring_bytes=0,
                 writer_threads=4, flags=MAPFILE, device=0, rank=0, world=1, nccl_unique_id=None, align=256,
                 pack_ctas=0, allreduce=None, allgather=None, d2h_gbs=0.0, d2h_quantum=0):
        """allreduce(values: list[int], is_max) -> list[int] and allgather(send, recv) replace the
        library's NCCL communicator when given (e.g. torch.distributed over gloo; see
        ``torch_collectives``).  allgather gets zero-copy numpy uint8 views of the library's pinned
        buffers — send (n bytes) and recv (world * n bytes, rank-ordered) — and fills recv in place,
        so no chunk bytes are copied through Python objects.
        d2h_gbs / d2h_quantum: pace the copy-engine D2H (GB/s, bytes per copy; 0 = unpaced)."""
        self._uid = None
        self._cbs = None
        ar = ag = None
        cbs = []
        if allreduce is not None:
            def _ar(ctx, vals, count, is_max):
                try:
                    out = allreduce([int(vals[i]) for i in range(count)], bool(is_max))
                    for i in range(count):
                        vals[i] = int(out[i])
                    return 0
                except Exception:  # noqa: BLE001
                    return 1
            cbs.append(ALLREDUCE_FN(_ar))
            ar = C.cast(cbs[-1], C.c_void_p)
        if allgather is not None:
            import numpy as np

            def _view(ptr, n):
                return np.ctypeslib.as_array(C.cast(ptr, C.POINTER(C.c_uint8)), shape=(n,)) if n else \
                    np.empty(0, dtype=np.uint8)

            def _ag(ctx, send, recv, nbytes):
                try:
                    allgather(_view(send, nbytes), _view(recv, nbytes * world))
                    return 0
                except Exception:  # noqa: BLE001
                    return 1
            cbs.append(ALLGATHER_FN(_ag))
            ag = C.cast(cbs[-1], C.c_void_p)
        self._cbs = cbs  # the C side holds raw pointers: keep the thunks alive
        if nccl_unique_id is not None:
            self._uid = C.create_string_buffer(bytes(nccl_unique_id), 128)
        self.cfg = Config(ABI_VERSION, path.encode() if path else None, chunk_bytes, max_inflight, staging_bytes,
                          ring_bytes, writer_threads, flags, device, rank, world,
                          C.cast(self._uid, C.c_void_p) if self._uid is not None else None, align, pack_ctas,
                          ar, ag, None, int(round(d2h_gbs * 1000)), int(d2h_quantum))
        self._ctx = C.c_void_p()
        _check(_lib.pcc_open(C.byref(self.cfg), C.byref(self._ctx)), "pcc_open")
        self._table = None

    def register(self, tensors, names=None):
        self._table, self._keep = tensor_table(tensors, names)
        _check(_lib.pcc_register(self._ctx, self._table, len(tensors)), "pcc_register")

    def checkpoint(self, it, stream=None):
        h = C.c_uint64()
        _check(_lib.pcc_checkpoint(self._ctx, it, _stream_ptr(stream), C.byref(h)), "pcc_checkpoint")
        return h.value

    def guard(self, stream=None):
        _check(_lib.pcc_guard(self._ctx, _stream_ptr(stream)), "pcc_guard")

    def poll(self, h):
        s = C.c_int()
        _check(_lib.pcc_poll(self._ctx, h, C.byref(s)), "pcc_poll")
        return s.value

    def wait(self, h, timeout_us=-1):
        _check(_lib.pcc_wait(self._ctx, h, timeout_us), "pcc_wait")

    def drain(self, timeout_us=-1):
        _check(_lib.pcc_drain(self._ctx, timeout_us), "pcc_drain")

    def commit(self):
        g = C.c_uint64()
        _check(_lib.pcc_commit(self._ctx, C.byref(g)), "pcc_commit")
        return None if g.value == NONE else g.value

    def restore(self, want_iter=None, fallback=False, bad_cap=4096):
        it = C.c_uint64()
        bad = (C.c_uint32 * bad_cap)()
        nbad = C.c_uint32()
        rc = _lib.pcc_restore(self._ctx, LATEST if want_iter is None else want_iter, FALLBACK if fallback else 0,
                              C.byref(it), bad, bad_cap, C.byref(nbad))
        bad_list = [bad[i] for i in range(min(nbad.value, bad_cap))]
        if rc != 0:
            err = PCCError(rc, "pcc_restore")
            err.bad_chunks = bad_list
            raise err
        return it.value, bad_list

    def restore_stats(self):
        """Where the last restore's time went (pcc_restore_stats): storage read, H2D, K2,
        finalize, fan-out (W > 1), total — ms, summed over the candidates tried."""
        r = RestoreInfo()
        _check(_lib.pcc_restore_stats(self._ctx, C.byref(r)), "pcc_restore_stats")
        return {f: getattr(r, f) for f, _ in RestoreInfo._fields_}

    def info(self, h, with_crc=False):
        inf = Info()
        n = self.geometry()["count"] if with_crc else 0
        crc = (C.c_uint32 * max(1, n))()
        _check(_lib.pcc_info(self._ctx, h, C.byref(inf), crc if with_crc else None, n), "pcc_info")
        d = {f: getattr(inf, f) for f, _ in Info._fields_}
        d["state_name"] = STATE_NAMES[inf.state]
        if with_crc:
            d["crc"] = [crc[i] for i in range(n)]
        return d

    def geometry(self):
        v = [C.c_uint64() for _ in range(4)]
        _check(_lib.pcc_geometry(self._ctx, *[C.byref(x) for x in v]), "pcc_geometry")
        return dict(n_chunks=v[0].value, first=v[1].value, count=v[2].value, end_bytes=v[3].value)

    def kernel_launches(self):
        return int(_lib.pcc_kernel_launches(self._ctx))

    def close(self):
        if self._ctx:
            _check(_lib.pcc_close(self._ctx), "pcc_close")
            self._ctx = C.c_void_p()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def torch_collectives(dist, group=None):
    """allreduce / allgather callbacks for ``PCCheck`` over an initialised torch.distributed
    CPU process group (gloo) — the transport for tests that run several ranks on one GPU, where
    NCCL cannot.  Marshalling only: allgather hands zero-copy tensors over the library's pinned
    buffers to ``dist.all_gather``."""
    import torch
    world = dist.get_world_size(group)

    def allreduce(vals, is_max):
        t = torch.tensor(vals, dtype=torch.int64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX if is_max else dist.ReduceOp.MIN, group=group)
        return t.tolist()

    def allgather(send, recv):
        st = torch.from_numpy(send)
        dist.all_gather(list(torch.from_numpy(recv).view(world, -1).unbind(0)), st, group=group)

    return dict(allreduce=allreduce, allgather=allgather)


_STATE_KEYS = ("momentum_buffer", "exp_avg", "exp_avg_sq", "step")


def state_tensors(optimizer, masters=None):
    """The registration list of reading R11 for a torch optimizer: per parameter
    in param-group order ``[param, (fp32 master), momentum_buffer | exp_avg, exp_avg_sq, step]``.
    ``masters`` maps a parameter to its fp32 master copy (mixed precision).  Returns
    ``(tensors, names)``; a state entry that is not a tensor (or lives on the host, e.g. the
    CPU ``step`` of non-fused Adam) raises — every registered tensor must be device memory."""
    import torch
    tensors, names = [], []
    k = 0
    for g in optimizer.param_groups:
        for p in g["params"]:
            entries = [("param", p.data)]
            if masters is not None and p in masters:
                entries.append(("master", masters[p]))
            st = optimizer.state.get(p, {})
            entries += [(key, st[key]) for key in _STATE_KEYS if key in st]
            for key, t in entries:
                if not isinstance(t, torch.Tensor) or (t.device.type != p.device.type):
                    raise ValueError(f"param {k} {key}: not a tensor on {p.device} (use fused/capturable optimizers)")
                tensors.append(t)
                names.append(f"{k}.{key}")
            k += 1
    return tensors, names


def latest(path):
    g, l = C.c_uint64(), C.c_uint64()
    rc = _lib.pcc_latest(path.encode(), C.byref(g), C.byref(l))
    if rc != 0:
        return None
    return g.value, l.value


def nccl_unique_id():
    buf = C.create_string_buffer(128)
    _check(_lib.pcc_nccl_unique_id(buf), "pcc_nccl_unique_id")
    return buf.raw


# ------------------------------------------------------------------- kernel-level calls
def nccl_selftest(vals, device=0):
    """The commit collective's NCCL calls on a one-rank communicator: (min, max, gather_ok)."""
    n = len(vals)
    v = (C.c_int64 * n)(*vals)
    mn, mx, ok = (C.c_int64 * n)(), (C.c_int64 * n)(), C.c_uint32()
    _check(_lib.pcc_k_nccl_selftest(device, v, n, mn, mx, C.byref(ok)), "pcc_k_nccl_selftest")
    return list(mn), list(mx), bool(ok.value)


def k_layout(tensors, align=256, chunk_bytes=4 << 20):
    tab, keep = tensor_table(tensors)
    n = len(tensors)
    off = (C.c_uint64 * max(1, n))()
    end, cnt = C.c_uint64(), C.c_uint64()
    _check(_lib.pcc_k_layout(tab, n, align, chunk_bytes, off, C.byref(end), C.byref(cnt)), "pcc_k_layout")
    return [off[i] for i in range(n)], end.value, cnt.value


def k_pack(tensors, dst_ptr, crc_ptr, digest_ptr, align=256, chunk_bytes=4 << 20, first_chunk=0, count=None,
           stream=None):
    """K1 into a caller buffer (device or host-mapped).  crc/digest are device pointers."""
    tab, keep = tensor_table(tensors)
    if count is None:
        count = k_layout(tensors, align, chunk_bytes)[2] - first_chunk
    _check(_lib.pcc_k_pack(tab, len(tensors), align, chunk_bytes, first_chunk, count, dst_ptr, crc_ptr, digest_ptr,
                           _stream_ptr(stream)), "pcc_k_pack")
    return count


def k_unpack(tensors, src_ptr, expect_ptr, bad_ptr, n_bad_ptr, digest_ptr, align=256, chunk_bytes=4 << 20,
             first_chunk=0, count=None, stream=None):
    """K2 from a caller buffer into the tensors (destinations)."""
    tab, keep = tensor_table(tensors)
    if count is None:
        count = k_layout(tensors, align, chunk_bytes)[2] - first_chunk
    _check(_lib.pcc_k_unpack(tab, len(tensors), align, chunk_bytes, first_chunk, count, src_ptr, expect_ptr,
                             bad_ptr, n_bad_ptr, digest_ptr, _stream_ptr(stream)), "pcc_k_unpack")
    return count


# -------------------------------------------------------------- commit engine (no GPU)
class HostEngine:
    """pccheck_host.h: Listing 1 + the DP commit rule over a rank file, without a GPU."""

    def __init__(self, path, chunk_bytes, max_inflight, rank, world, total_chunks, n_tensors=0, align=256,
                 layout_crc=0, fsync=False):
        cfg = HostConfig(path.encode() if path else None, chunk_bytes, max_inflight, rank, world, total_chunks,
                         n_tensors, align, layout_crc, 1 if fsync else 0)
        self._h = C.c_void_p()
        _check(_lib.pcc_host_open(C.byref(cfg), C.byref(self._h)), "pcc_host_open")

    def begin(self, it):
        c, s = C.c_uint64(), C.c_uint32()
        rc = _lib.pcc_host_begin(self._h, it, C.byref(c), C.byref(s))
        if rc == -EAGAIN:
            return None
        _check(rc, "pcc_host_begin")
        return c.value, s.value

    def filling(self, counter):
        _check(_lib.pcc_host_filling(self._h, counter), "pcc_host_filling")

    def complete(self, counter, crcs, digest):
        arr = (C.c_uint32 * max(1, len(crcs)))(*crcs)
        st = C.c_int()
        _check(_lib.pcc_host_complete(self._h, counter, arr, digest, C.byref(st)), "pcc_host_complete")
        return st.value

    def fail(self, counter):
        _check(_lib.pcc_host_fail(self._h, counter), "pcc_host_fail")

    def state(self, counter):
        st = C.c_int()
        _check(_lib.pcc_host_state(self._h, counter, C.byref(st)), "pcc_host_state")
        return st.value

    def local_latest(self):
        v = _lib.pcc_host_local_latest(self._h)
        return None if v == NONE else v

    def global_iter(self):
        v = _lib.pcc_host_global(self._h)
        return None if v == NONE else v

    def apply_global(self, g):
        _check(_lib.pcc_host_apply_global(self._h, g), "pcc_host_apply_global")

    def free_slots(self):
        return int(_lib.pcc_host_free_slots(self._h))

    def geometry(self):
        a, b, c = C.c_uint32(), C.c_uint32(), C.c_uint32()
        _lib.pcc_host_geometry(self._h, C.byref(a), C.byref(b), C.byref(c))
        return a.value, b.value, c.value

    def data_offset(self, slot):
        return int(_lib.pcc_host_data_offset(self._h, slot))

    def held(self):
        it = (C.c_uint64 * 64)()
        sl = (C.c_uint32 * 64)()
        k = _lib.pcc_host_held(self._h, it, sl, 64)
        return {it[i]: sl[i] for i in range(min(k, 64))}

    def restore_plan(self, reduce, verify, want_iter=None, fallback=False):
        """reduce(value:int, is_max:bool) -> int (an allreduce across ranks); verify(iter, slot) -> bool."""
        def _r(ctx, v, is_max):
            v[0] = int(reduce(int(v[0]), bool(is_max)))
            return 0

        def _v(ctx, it, slot):
            return 0 if verify(int(it), int(slot)) else 1

        rf, vf = REDUCE_FN(_r), VERIFY_FN(_v)
        out = C.c_uint64()
        rc = _lib.pcc_host_restore_plan(self._h, LATEST if want_iter is None else want_iter,
                                        FALLBACK if fallback else 0, C.cast(rf, C.c_void_p), C.cast(vf, C.c_void_p),
                                        None, C.byref(out))
        if rc != 0:
            raise PCCError(rc, "pcc_host_restore_plan")
        return out.value

    def close(self):
        if self._h:
            _lib.pcc_host_close(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
