"""Thin ctypes binding of libmstamp_b200.so (include/mp.h).

Argument marshalling only: every step of the method runs in the CUDA kernels
behind the C ABI.  There is no CPU fallback -- ``load()`` raises if the shared
library is missing or no CUDA device is usable.

Host-memory entry point: ``Context.compute(T, m, ...)`` (numpy in/out, includes
the H2D/D2H copies).  Device entry points take torch CUDA tensors (torch is used
only for device memory, streams and process groups).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("MP_LIB_PATH") or os.path.join(_HERE, "lib", "libmstamp_b200.so")

PRECISIONS = {"fp64": 0, "fp32": 1, "fp16": 2, "mixed": 3, "fp16c": 4, "fp16ck": 5}
STATUS = {0: "MP_OK", 1: "MP_ERR_INVALID", 2: "MP_ERR_NOMEM", 3: "MP_ERR_CUDA", 4: "MP_ERR_NCCL",
          5: "MP_ERR_UNSUPPORTED"}
EXPORTS = ["mp_init", "mp_free", "mp_last_error", "mp_version", "mp_compute", "mp_compute_device",
           "mp_key_words", "mp_partial_device", "mp_key_mask_device", "mp_finalize_device",
           "mp_plan_bands", "mp_plan_diagonals", "mp_last_timing", "mp_selftest_sort_scan",
           "mp_selftest_precompute", "mp_compute_stream", "mp_plan_stream", "mp_last_stream_info",
           "mp_selftest_seeds"]

_lib = None


class MPError(RuntimeError):
    def __init__(self, status, msg=""):
        self.status = status
        super().__init__(f"{STATUS.get(status, status)}: {msg}")


class _Config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("reseed_h", ctypes.c_int64 * 4), ("seed_mode", ctypes.c_int)]


SEED_MODES = {"direct": 0, "tc": 1}   # mp_config.seed_mode (MP_SEEDS_DIRECT / MP_SEEDS_TC)


def load():
    """Load the C-ABI library (fails loudly if it was not built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build() (no CPU fallback exists)")
    lib = ctypes.CDLL(LIB_PATH)
    i64, p, i32 = ctypes.c_int64, ctypes.c_void_p, ctypes.c_int
    lib.mp_init.argtypes = [ctypes.POINTER(p), ctypes.POINTER(_Config)]
    lib.mp_init.restype = i32
    lib.mp_free.argtypes = [p]
    lib.mp_free.restype = None
    lib.mp_last_error.argtypes = [p]
    lib.mp_last_error.restype = ctypes.c_char_p
    lib.mp_version.argtypes = []
    lib.mp_version.restype = ctypes.c_char_p
    lib.mp_compute.argtypes = [p, p, p, i64, i64, i64, i32, i64, p, p]
    lib.mp_compute.restype = i32
    lib.mp_compute_device.argtypes = [p, p, p, p, i64, i64, i64, i32, i64, p, p]
    lib.mp_compute_device.restype = i32
    lib.mp_key_words.argtypes = [i64, i64, i32]
    lib.mp_key_words.restype = i64
    lib.mp_partial_device.argtypes = [p, p, p, p, i64, i64, i64, i32, i64, i32, i32, p]
    lib.mp_partial_device.restype = i32
    lib.mp_key_mask_device.argtypes = [p, p, i64, i64, p, p]
    lib.mp_key_mask_device.restype = i32
    lib.mp_finalize_device.argtypes = [p, p, i64, i64, i32, p, p, p]
    lib.mp_finalize_device.restype = i32
    lib.mp_plan_bands.argtypes = [i64, i64, i64, i32, i64, i32, i32, p, p]
    lib.mp_plan_bands.restype = i32
    lib.mp_plan_diagonals.argtypes = [i64, i64, i64, i32, i64, i32, i32, p]
    lib.mp_plan_diagonals.restype = i32
    lib.mp_last_timing.argtypes = [p, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(i64)]
    lib.mp_last_timing.restype = i32
    lib.mp_selftest_sort_scan.argtypes = [p, i64, i64, p, p]
    lib.mp_selftest_sort_scan.restype = i32
    lib.mp_selftest_precompute.argtypes = [p, p, i64, i64, i64, i32, p, p, p]
    lib.mp_selftest_precompute.restype = i32
    optional = {  # absent from libraries built before round 2 (MP_LIB_PATH variants)
        "mp_selftest_seeds": [p, p, p, i64, i64, i64, i32, i64, i64, i64, p, p],
        "mp_compute_stream": [p, p, p, i64, i64, i64, i32, i64, i64, p, p],
        "mp_plan_stream": [i64, i64, i64, i32, i64, i32, i64, i64, p, p],
        "mp_last_stream_info": [p, p, p, p, p],
    }
    for name, args in optional.items():
        if hasattr(lib, name):
            getattr(lib, name).argtypes = args
            getattr(lib, name).restype = i32
    _lib = lib
    return lib


def _prec(prec):
    if isinstance(prec, str):
        return PRECISIONS[prec.lower()]
    return int(prec)


def version() -> str:
    return load().mp_version().decode()


def plan_bands(d, n, m, prec="fp32", exclusion=-1, self_join=True, world=1):
    """Host scheduler: (block_begin[world+1], cells[world]) of the equal-cell diagonal bands."""
    lib = load()
    bb = np.zeros(world + 1, dtype=np.int64)
    cells = np.zeros(world, dtype=np.int64)
    st = lib.mp_plan_bands(d, n, m, _prec(prec), exclusion, int(bool(self_join)), world,
                           bb.ctypes.data_as(ctypes.c_void_p), cells.ctypes.data_as(ctypes.c_void_p))
    if st != 0:
        raise MPError(st, "mp_plan_bands")
    return bb, cells


def plan_diagonals(d, n, m, prec="fp32", exclusion=-1, self_join=True, world=1):
    """Host scheduler: band g covers diagonals [diag_begin[g], diag_begin[g+1])."""
    lib = load()
    db = np.zeros(world + 1, dtype=np.int64)
    st = lib.mp_plan_diagonals(d, n, m, _prec(prec), exclusion, int(bool(self_join)), world,
                               db.ctypes.data_as(ctypes.c_void_p))
    if st != 0:
        raise MPError(st, "mp_plan_diagonals")
    return db


def plan_stream(d, n, m, prec="fp32", exclusion=-1, self_join=True, device_bytes=1 << 30,
                granularity=2 << 20):
    """Host scheduler of mp_compute_stream: (rows per chunk R, diagonals per band Wb)."""
    lib = load()
    out = np.zeros(2, dtype=np.int64)
    st = lib.mp_plan_stream(d, n, m, _prec(prec), exclusion, int(bool(self_join)), int(device_bytes),
                            int(granularity), out[0:].ctypes.data_as(ctypes.c_void_p),
                            out[1:].ctypes.data_as(ctypes.c_void_p))
    if st != 0:
        raise MPError(st, "mp_plan_stream")
    return int(out[0]), int(out[1])


def key_words(d, n, prec="fp32") -> int:
    return int(load().mp_key_words(d, n, _prec(prec)))


def _tptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _need(t, name, dtype, device, shape=None, min_numel=None):
    """Argument marshalling guard: a torch tensor of the dtype, on the context's device,
    contiguous and of the shape the C ABI reads or writes (else MPError(MP_ERR_INVALID) before
    any device pointer crosses the boundary)."""
    import torch
    if not isinstance(t, torch.Tensor):
        raise MPError(1, f"{name} must be a torch tensor")
    if t.dtype != dtype:
        raise MPError(1, f"{name} must be {dtype}, got {t.dtype}")
    if t.device.type != "cuda" or t.device.index != device:
        raise MPError(1, f"{name} must live on cuda:{device}, got {t.device}")
    if not t.is_contiguous():
        raise MPError(1, f"{name} must be contiguous")
    if shape is not None and tuple(t.shape) != tuple(shape):
        raise MPError(1, f"{name} must have shape {tuple(shape)}, got {tuple(t.shape)}")
    if min_numel is not None and t.numel() < min_numel:
        raise MPError(1, f"{name} needs >= {min_numel} elements, has {t.numel()}")


class Context:
    """One context per host thread / GPU (mp_init ... mp_free)."""

    def __init__(self, device: int = 0, reseed_h=None, seed_mode="direct"):
        lib = load()
        cfg = _Config()
        cfg.device = device
        cfg.seed_mode = SEED_MODES[seed_mode] if isinstance(seed_mode, str) else int(seed_mode)
        h = list(reseed_h or [0, 0, 0, 0])
        for i in range(4):
            cfg.reseed_h[i] = int(h[i])
        self._ctx = ctypes.c_void_p()
        st = lib.mp_init(ctypes.byref(self._ctx), ctypes.byref(cfg))
        if st != 0:
            raise MPError(st, "mp_init")
        self.device = device

    def close(self):
        if self._ctx:
            load().mp_free(self._ctx)
            self._ctx = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, st, what):
        if st != 0:
            raise MPError(st, f"{what}: {load().mp_last_error(self._ctx).decode()}")

    # ---- host memory
    def compute(self, T, m, prec="fp32", exclusion=-1, Tr=None, out=None):
        """P (d,n) float64 and I (d,n) int64 from host series T (d,L) [and Tr].

        out: optional preallocated (P, I) host arrays (C-contiguous float64 / int64, shape
        (d, n)), e.g. views of pinned buffers, so repeated calls skip the allocation and the
        page faults of fresh output memory."""
        T = np.ascontiguousarray(T, dtype=np.float64)
        if T.ndim == 1:
            T = T[None, :]
        d, L = T.shape
        n = L - m + 1
        Tr_ = None
        if Tr is not None:
            Tr_ = np.ascontiguousarray(Tr, dtype=np.float64)
            if Tr_.ndim == 1:
                Tr_ = Tr_[None, :]
            if Tr_.shape != T.shape:
                raise MPError(1, "AB-join needs equal shapes")
        if out is None:
            P = np.empty((d, n), dtype=np.float64)
            I = np.empty((d, n), dtype=np.int64)
        else:
            P, I = out
            if (P.shape != (d, n) or I.shape != (d, n) or P.dtype != np.float64 or I.dtype != np.int64
                    or not P.flags.c_contiguous or not I.flags.c_contiguous):
                raise MPError(1, "out must be C-contiguous float64 / int64 arrays of shape (d, n)")
        st = load().mp_compute(self._ctx, T.ctypes.data_as(ctypes.c_void_p),
                               None if Tr_ is None else Tr_.ctypes.data_as(ctypes.c_void_p),
                               d, n, m, _prec(prec), int(exclusion),
                               P.ctypes.data_as(ctypes.c_void_p), I.ctypes.data_as(ctypes.c_void_p))
        self._check(st, "mp_compute")
        return P, I

    def compute_stream(self, T, m, prec="fp32", exclusion=-1, Tr=None, device_bytes=1 << 30, out=None):
        """Beyond-memory streaming (mp_compute_stream): the same P, I as compute() with at most
        about device_bytes of device memory for the per-position arrays."""
        T = np.ascontiguousarray(T, dtype=np.float64)
        if T.ndim == 1:
            T = T[None, :]
        d, L = T.shape
        n = L - m + 1
        Tr_ = None
        if Tr is not None:
            Tr_ = np.ascontiguousarray(Tr, dtype=np.float64)
            if Tr_.ndim == 1:
                Tr_ = Tr_[None, :]
            if Tr_.shape != T.shape:
                raise MPError(1, "AB-join needs equal shapes")
        if out is None:
            P = np.empty((d, n), dtype=np.float64)
            I = np.empty((d, n), dtype=np.int64)
        else:
            P, I = out
            if (P.shape != (d, n) or I.shape != (d, n) or P.dtype != np.float64 or I.dtype != np.int64
                    or not P.flags.c_contiguous or not I.flags.c_contiguous):
                raise MPError(1, "out must be C-contiguous float64 / int64 arrays of shape (d, n)")
        st = load().mp_compute_stream(self._ctx, T.ctypes.data_as(ctypes.c_void_p),
                                      None if Tr_ is None else Tr_.ctypes.data_as(ctypes.c_void_p),
                                      d, n, m, _prec(prec), int(exclusion), int(device_bytes),
                                      P.ctypes.data_as(ctypes.c_void_p), I.ctypes.data_as(ctypes.c_void_p))
        self._check(st, "mp_compute_stream")
        return P, I

    def last_stream_info(self):
        """(rows per chunk, diagonals per band, peak mapped device bytes, launches) of the last
        compute_stream."""
        v = np.zeros(4, dtype=np.int64)
        ptr = [ctypes.c_void_p(v.ctypes.data + 8 * k) for k in range(4)]
        self._check(load().mp_last_stream_info(self._ctx, *ptr), "mp_last_stream_info")
        return tuple(int(x) for x in v)

    # ---- device memory (torch tensors)
    def compute_device(self, T, m, P, I, prec="fp32", exclusion=-1, Tr=None, stream=None):
        import torch
        _need(T, "T", torch.float64, self.device)
        d, L = T.shape
        n = L - m + 1
        if Tr is not None:
            _need(Tr, "Tr", torch.float64, self.device, shape=T.shape)
        _need(P, "P", torch.float64, self.device, shape=(d, n))
        _need(I, "I", torch.int64, self.device, shape=(d, n))
        s = stream if stream is not None else torch.cuda.current_stream(T.device)
        st = load().mp_compute_device(self._ctx, ctypes.c_void_p(s.cuda_stream), _tptr(T), _tptr(Tr),
                                      d, n, m, _prec(prec), int(exclusion), _tptr(P), _tptr(I))
        self._check(st, "mp_compute_device")

    def partial_device(self, T, m, keys, rank, world, prec="fp32", exclusion=-1, Tr=None, stream=None):
        import torch
        _need(T, "T", torch.float64, self.device)
        d, L = T.shape
        n = L - m + 1
        if Tr is not None:
            _need(Tr, "Tr", torch.float64, self.device, shape=T.shape)
        _need(keys, "keys", torch.int64, self.device, min_numel=key_words(d, n, prec))
        s = stream if stream is not None else torch.cuda.current_stream(T.device)
        st = load().mp_partial_device(self._ctx, ctypes.c_void_p(s.cuda_stream), _tptr(T), _tptr(Tr),
                                      d, n, m, _prec(prec), int(exclusion), int(rank), int(world),
                                      _tptr(keys))
        self._check(st, "mp_partial_device")

    def key_mask_device(self, d, n, keys, global_v, stream=None):
        import torch
        _need(keys, "keys", torch.int64, self.device, min_numel=2 * d * n)
        _need(global_v, "global_v", torch.int64, self.device, min_numel=d * n)
        s = stream if stream is not None else torch.cuda.current_stream(keys.device)
        st = load().mp_key_mask_device(self._ctx, ctypes.c_void_p(s.cuda_stream), d, n, _tptr(keys),
                                       _tptr(global_v))
        self._check(st, "mp_key_mask_device")

    def finalize_device(self, d, n, keys, P, I, prec="fp32", stream=None):
        import torch
        _need(keys, "keys", torch.int64, self.device, min_numel=key_words(d, n, prec))
        _need(P, "P", torch.float64, self.device, shape=(d, n))
        _need(I, "I", torch.int64, self.device, shape=(d, n))
        s = stream if stream is not None else torch.cuda.current_stream(keys.device)
        st = load().mp_finalize_device(self._ctx, ctypes.c_void_p(s.cuda_stream), d, n, _prec(prec),
                                       _tptr(keys), _tptr(P), _tptr(I))
        self._check(st, "mp_finalize_device")

    # ---- stage self-tests (include/mp.h; tests only)
    def selftest_sort_scan(self, X):
        """X (count, d) float32 -> inclusive prefix sums of each row sorted ascending, computed by
        the FP32 kernels' own sort / merge / scan device code for this d."""
        X = np.ascontiguousarray(X, dtype=np.float32)
        count, d = X.shape
        out = np.empty_like(X)
        st = load().mp_selftest_sort_scan(self._ctx, d, count, X.ctypes.data_as(ctypes.c_void_p),
                                          out.ctypes.data_as(ctypes.c_void_p))
        self._check(st, "mp_selftest_sort_scan")
        return out

    def selftest_precompute(self, T, m, prec="fp64"):
        """(df, dg, a), each (n, d) position-major, from the device precalculation of mode prec."""
        T = np.ascontiguousarray(T, dtype=np.float64)
        d, L = T.shape
        n = L - m + 1
        outs = [np.empty((n, d)) for _ in range(3)]
        st = load().mp_selftest_precompute(self._ctx, T.ctypes.data_as(ctypes.c_void_p), d, n, m, _prec(prec),
                                           *[o.ctypes.data_as(ctypes.c_void_p) for o in outs])
        self._check(st, "mp_selftest_precompute")
        return tuple(outs)

    def selftest_seeds(self, T, m, prec="mixed", H=256, rows=(0, 1), Tr=None):
        """Tensor-core seed table (MP_SEEDS_TC) of re-seed rows r*H, r in [rows[0], rows[1]), against
        every column: ((r, d, n) doubles in the precalc's scaled units, per-dimension scales)."""
        T = np.ascontiguousarray(T, dtype=np.float64)
        d, L = T.shape
        n = L - m + 1
        Tr_ = None if Tr is None else np.ascontiguousarray(Tr, dtype=np.float64)
        r0, r1 = rows
        out = np.empty((r1 - r0, d, n))
        sc = np.zeros(2 * d)
        st = load().mp_selftest_seeds(self._ctx, T.ctypes.data_as(ctypes.c_void_p),
                                      None if Tr_ is None else Tr_.ctypes.data_as(ctypes.c_void_p),
                                      d, n, m, _prec(prec), H, r0, r1, out.ctypes.data_as(ctypes.c_void_p),
                                      sc.ctypes.data_as(ctypes.c_void_p))
        self._check(st, "mp_selftest_seeds")
        return out, (sc[:d] if Tr is None else sc)

    def last_timing(self):
        ms = ctypes.c_double()
        nl = ctypes.c_int64()
        self._check(load().mp_last_timing(self._ctx, ctypes.byref(ms), ctypes.byref(nl)), "mp_last_timing")
        return ms.value, nl.value


def merge_partials(ctx: Context, keys, d, n, prec, group=None, mask=None):
    """MINLOC all-reduce of partial keys over the process group (the path's one exchange).

    FP32/FP16/MIXED: one int64 MIN.  FP64: MIN on the value plane, mask indices whose
    value lost (mp_key_mask_device), MIN on the index plane.  ``keys`` is
    modified in place.  ``mask`` overrides the mask step (CPU protocol tests only).
    """
    import torch.distributed as dist
    count = d * n
    if _prec(prec) == 0:
        v = keys[:count]
        gv = v.clone()
        dist.all_reduce(gv, op=dist.ReduceOp.MIN, group=group)
        if mask is None:
            ctx.key_mask_device(d, n, keys, gv)
        else:
            mask(keys, gv)
        v.copy_(gv)
        dist.all_reduce(keys[count:], op=dist.ReduceOp.MIN, group=group)
    else:
        dist.all_reduce(keys, op=dist.ReduceOp.MIN, group=group)
    return keys
