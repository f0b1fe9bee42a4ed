"""Thin Python binding of libmsm.so (include/msm.h): argument marshalling only.

Every step of the MSM runs in the library's CUDA kernels; this module converts numpy /
torch buffers to pointers and return codes to exceptions.  It fails loudly when the
shared library is missing (there is no CPU fallback).

    ctx = Context("bls12_381", points, ngpus=1)   # points: [n, 2*L32] uint32 words
    x, y = ctx.run(scalars)                       # scalars: [n, S] uint32 words -> ints
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_LIB = None
_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("MSM_LIB") or os.path.join(_HERE, "libmsm.so")  # MSM_LIB: A/B variant builds

CURVE_IDS = {"bn254": 0, "bls12_377": 1, "bls12_381": 2, "mnt4_753": 3}

OPT_WINDOW_BITS = 1
OPT_ACC_THREADS = 2
OPT_SEG_LEN = 3
OPT_SORT = 4
OPT_PRECOMPUTE = 5
OPT_SPLIT_PARTS = 6
OPT_SPLIT_INDEX = 7
OPT_ACC_MODE = 8
OPT_H2D_CHUNKS = 9
OPT_GRAPH = 10
OPT_NWIN = 101
OPT_NONEMPTY = 102
OPT_NSETS = 103
OPT_DEVICE = 104
OPT_NGPUS = 105

ERRORS = {
    0: "ok", -1: "invalid argument", -2: "unknown curve", -3: "CUDA error", -4: "device out of memory",
    -5: "NCCL error", -6: "point not on curve or not canonical", -7: "scalar >= r", -8: "unimplemented",
    -9: "no (or not enough) CUDA devices",
}


class MSMError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        self.code = code
        super().__init__(f"{what}: {ERRORS.get(code, 'error')} ({code})" if what else f"{ERRORS.get(code, 'error')} ({code})")


class Stats(ctypes.Structure):
    _fields_ = [
        ("h2d_ms", ctypes.c_float), ("sort_ms", ctypes.c_float), ("accumulate_ms", ctypes.c_float),
        ("fixup_ms", ctypes.c_float), ("reduce_ms", ctypes.c_float), ("combine_ms", ctypes.c_float),
        ("finalize_ms", ctypes.c_float), ("total_ms", ctypes.c_float), ("window_bits", ctypes.c_int),
        ("nwin", ctypes.c_int), ("acc_threads", ctypes.c_int), ("acc_launches", ctypes.c_int),
        ("entries", ctypes.c_uint64), ("precompute", ctypes.c_int), ("table_ms", ctypes.c_float),
        ("baff_ms", ctypes.c_float), ("baff", ctypes.c_int), ("entries_acc", ctypes.c_uint64),
    ]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


def lib() -> ctypes.CDLL:
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run `python tools/build.py` (or __graft_entry__.build())")
    L = ctypes.CDLL(LIB_PATH)
    P = ctypes.c_void_p
    sz = ctypes.c_size_t
    i = ctypes.c_int
    sig = {
        "msm_field_words": (i, [i]), "msm_scalar_words": (i, [i]), "msm_scalar_bits": (i, [i]),
        "msm_partial_words": (i, [i]), "msm_device_count": (i, []),
        "msm_context_create": (P, [i, P, sz, i]), "msm_context_destroy": (None, [P]),
        "msm_context_create_on": (P, [i, P, sz, i, P]),
        "msm_shard_info": (i, [P, i, P, P, P]),
        "msm_run": (i, [P, P, P]), "msm_run_partial": (i, [P, P, P]), "msm_finalize": (i, [i, P, i, P]),
        "msm_submit": (ctypes.c_long, [P, P]), "msm_wait": (i, [P, ctypes.c_long, P]),
        "msm_set_option": (i, [P, i, ctypes.c_long]), "msm_get_option": (ctypes.c_long, [P, i]),
        "msm_get_stats": (i, [P, ctypes.POINTER(Stats)]), "msm_get_stream": (P, [P, i]),
        "msm_last_error": (i, []), "msm_error_string": (ctypes.c_char_p, [i]),
        "msm_gen_points": (i, [i, P, P, sz, P]),
        "msm_debug_field": (i, [i, i, P, P, sz, P]), "msm_debug_ec": (i, [i, i, P, P, P, sz, P]),
        "msm_debug_digits": (i, [i, i, P, sz, P]), "msm_debug_windows": (i, [P, P, P, P]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _LIB = L
    return L


def curve_id(curve) -> int:
    if isinstance(curve, int):
        return curve
    return CURVE_IDS[curve]


def field_words(curve) -> int:
    return lib().msm_field_words(curve_id(curve))


def scalar_words(curve) -> int:
    return lib().msm_scalar_words(curve_id(curve))


def partial_words(curve) -> int:
    return lib().msm_partial_words(curve_id(curve))


def device_count() -> int:
    return lib().msm_device_count()


def _check(rc: int, what: str):
    if rc != 0:
        raise MSMError(rc, what)


def _ptr(buf, dtype=np.uint32, words=None):
    """(pointer, keepalive) for a numpy array or torch tensor of 32-bit words."""
    if buf is None:
        return None, None
    if hasattr(buf, "data_ptr"):  # torch tensor (CPU or CUDA), int32/uint32 words
        if not buf.is_contiguous():
            raise ValueError("tensor must be contiguous")
        if buf.element_size() != 4:
            raise ValueError("tensor must hold 32-bit words")
        if words is not None and buf.numel() < words:
            raise ValueError(f"buffer too small: {buf.numel()} < {words} words")
        return ctypes.c_void_p(buf.data_ptr()), buf
    a = np.ascontiguousarray(buf)
    if a.dtype.itemsize != 4:
        a = a.astype(dtype)
    if words is not None and a.size < words:
        raise ValueError(f"buffer too small: {a.size} < {words} words")
    return ctypes.c_void_p(a.ctypes.data), a


def words_to_int(ws) -> int:
    return int.from_bytes(np.asarray(ws, dtype=np.uint32).tobytes(), "little")


def point_from_words(ws, L32):
    ws = np.asarray(ws, dtype=np.uint32)
    return words_to_int(ws[:L32]), words_to_int(ws[L32:2 * L32])


class Context:
    """A set of fixed points resident on `ngpus` devices (msm_context_create)."""

    def __init__(self, curve, points, ngpus: int = 1, n: int | None = None, devices=None):
        """devices: optional CUDA device per shard (msm_context_create_on; a device may
        repeat: logical shards on one GPU).  Default: shards on the current device onward."""
        self.curve = curve_id(curve)
        self.L32 = field_words(self.curve)
        self.S = scalar_words(self.curve)
        if n is None:
            n = (points.numel() if hasattr(points, "numel") else np.asarray(points).size) // (2 * self.L32)
        self.n = n
        p, keep = _ptr(points, words=n * 2 * self.L32) if n else (None, None)
        if devices is not None:
            ngpus = len(devices)
            dv = (ctypes.c_int * ngpus)(*devices)
            h = lib().msm_context_create_on(self.curve, p, n, ngpus, ctypes.cast(dv, ctypes.c_void_p))
        else:
            h = lib().msm_context_create(self.curve, p, n, ngpus)
        if not h:
            raise MSMError(lib().msm_last_error(), "msm_context_create")
        self._h = ctypes.c_void_p(h)
        self.ngpus = ngpus

    def shard_info(self, g: int):
        """(device, offset, count) of shard g."""
        d = ctypes.c_int()
        off = ctypes.c_size_t()
        cnt = ctypes.c_size_t()
        _check(lib().msm_shard_info(self._h, g, ctypes.byref(d), ctypes.byref(off), ctypes.byref(cnt)), "msm_shard_info")
        return d.value, off.value, cnt.value

    def close(self):
        if getattr(self, "_h", None):
            lib().msm_context_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def run_words(self, scalars, out=None) -> np.ndarray:
        """Q as 2*L32 canonical words (x then y); (0, 0) = O."""
        res = np.zeros(2 * self.L32, dtype=np.uint32) if out is None else out
        sp, keep = _ptr(scalars, words=self.n * self.S) if self.n else (None, None)
        _check(lib().msm_run(self._h, sp, ctypes.c_void_p(res.ctypes.data)), "msm_run")
        return res

    def run(self, scalars):
        """Q = sum k_i P_i as affine ints (x, y); O -> (0, 0)."""
        return point_from_words(self.run_words(scalars), self.L32)

    def submit(self, scalars) -> int:
        """Pipelined MSM (msm_submit): enqueue and return a ticket; the scalar buffer is kept
        alive here until wait(ticket)."""
        sp, keep = _ptr(scalars, words=self.n * self.S) if self.n else (None, None)
        t = lib().msm_submit(self._h, sp)
        if t < 0:
            raise MSMError(int(t), "msm_submit")
        if not hasattr(self, "_inflight"):
            self._inflight = {}
        self._inflight[t] = keep
        return t

    def wait_words(self, ticket: int, out=None) -> np.ndarray:
        res = np.zeros(2 * self.L32, dtype=np.uint32) if out is None else out
        try:
            _check(lib().msm_wait(self._h, ticket, ctypes.c_void_p(res.ctypes.data)), "msm_wait")
        finally:
            getattr(self, "_inflight", {}).pop(ticket, None)
        return res

    def wait(self, ticket: int):
        """Result of a submitted MSM as affine ints (x, y)."""
        return point_from_words(self.wait_words(ticket), self.L32)

    def run_partial(self, scalars, out):
        sp, keep = _ptr(scalars, words=self.n * self.S) if self.n else (None, None)
        op, keep2 = _ptr(out, words=partial_words(self.curve))
        _check(lib().msm_run_partial(self._h, sp, op), "msm_run_partial")
        return out

    def windows(self, scalars, with_buckets=False):
        """Debug: per-set sums W_s = sum_b b*B_{s,b} (and bucket sums B_{s,b}) as affine int
        pairs.  Without the f3 table the sets are the windows j; with it there is one set."""
        nwin = self.get_option(OPT_NSETS)
        c = self.get_option(OPT_WINDOW_BITS)
        W = np.zeros(nwin * 2 * self.L32, dtype=np.uint32)
        B = np.zeros(nwin * ((1 << (c - 1)) + 1) * 2 * self.L32, dtype=np.uint32) if with_buckets else None
        sp, keep = _ptr(scalars, words=self.n * self.S) if self.n else (None, None)
        _check(lib().msm_debug_windows(self._h, sp, ctypes.c_void_p(W.ctypes.data),
                                       ctypes.c_void_p(B.ctypes.data) if B is not None else None), "msm_debug_windows")
        Ws = [point_from_words(W[j * 2 * self.L32:(j + 1) * 2 * self.L32], self.L32) for j in range(nwin)]
        if not with_buckets:
            return Ws
        nb = (1 << (c - 1)) + 1
        Bs = [[point_from_words(B[(j * nb + b) * 2 * self.L32:(j * nb + b + 1) * 2 * self.L32], self.L32)
               for b in range(nb)] for j in range(nwin)]
        return Ws, Bs

    def set_option(self, key: int, value: int):
        _check(lib().msm_set_option(self._h, key, value), "msm_set_option")

    def get_option(self, key: int) -> int:
        return lib().msm_get_option(self._h, key)

    def stats(self) -> dict:
        s = Stats()
        _check(lib().msm_get_stats(self._h, ctypes.byref(s)), "msm_get_stats")
        return s.as_dict()

    def stream(self, dev: int = 0) -> int:
        return lib().msm_get_stream(self._h, dev) or 0


def finalize(curve, partials, count: int):
    """Sum `count` XYZZ partials (host or device words) -> affine ints (x, y)."""
    cid = curve_id(curve)
    L32 = field_words(cid)
    res = np.zeros(2 * L32, dtype=np.uint32)
    pp, keep = _ptr(partials, words=count * partial_words(cid))
    _check(lib().msm_finalize(cid, pp, count, ctypes.c_void_p(res.ctypes.data)), "msm_finalize")
    return point_from_words(res, L32)


def gen_points(curve, e0: int, delta: int, n: int, out):
    """P_i = (e0 + i*delta) G into the device tensor `out` ([n, 2*L32] 32-bit words)."""
    cid = curve_id(curve)
    S = scalar_words(cid)
    e = np.array([(e0 >> (32 * i)) & 0xFFFFFFFF for i in range(S)], dtype=np.uint32)
    d = np.array([(delta >> (32 * i)) & 0xFFFFFFFF for i in range(S)], dtype=np.uint32)
    op, keep = _ptr(out, words=n * 2 * field_words(cid))
    _check(lib().msm_gen_points(cid, ctypes.c_void_p(e.ctypes.data), ctypes.c_void_p(d.ctypes.data), n, op),
           "msm_gen_points")
    return out


def debug_field(curve, op: int, a: np.ndarray, b: np.ndarray) -> np.ndarray:
    cid = curve_id(curve)
    a = np.ascontiguousarray(a, dtype=np.uint32)
    b = np.ascontiguousarray(b, dtype=np.uint32)
    n = a.shape[0]
    out = np.zeros_like(a)
    _check(lib().msm_debug_field(cid, op, ctypes.c_void_p(a.ctypes.data), ctypes.c_void_p(b.ctypes.data), n,
                                 ctypes.c_void_p(out.ctypes.data)), "msm_debug_field")
    return out


def debug_ec(curve, op: int, P: np.ndarray, Q: np.ndarray, z: np.ndarray) -> np.ndarray:
    cid = curve_id(curve)
    P, Q, z = (np.ascontiguousarray(v, dtype=np.uint32) for v in (P, Q, z))
    n = P.shape[0]
    out = np.zeros_like(P)
    _check(lib().msm_debug_ec(cid, op, ctypes.c_void_p(P.ctypes.data), ctypes.c_void_p(Q.ctypes.data),
                              ctypes.c_void_p(z.ctypes.data), n, ctypes.c_void_p(out.ctypes.data)), "msm_debug_ec")
    return out


def debug_digits(curve, c: int, scalars: np.ndarray) -> np.ndarray:
    cid = curve_id(curve)
    s = np.ascontiguousarray(scalars, dtype=np.uint32)
    n = s.shape[0]
    nwin = lib().msm_scalar_bits(cid) // c + 1
    out = np.zeros((n, nwin), dtype=np.int32)
    _check(lib().msm_debug_digits(cid, c, ctypes.c_void_p(s.ctypes.data), n, ctypes.c_void_p(out.ctypes.data)),
           "msm_debug_digits")
    return out
