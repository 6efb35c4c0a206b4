"""CPU oracle of the PFPL codec -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this module.  The
product path (``paper_conf_ipps_fallinadcb25_b200``) never imports it and
shares no code with it.  The arithmetic lives in ``pfpl_oracle.c`` (plain C,
written step by step from /root/reference/PAPER.md, see its header for the
citations); this file only marshals numpy arrays through ctypes.

Parity status: pinned by tests/test_oracle_*.py,
except the bit patterns of the log2p/pow2p coefficients, whose *accuracy*
is pinned but whose exact values are format constants ("parity unpinned"
for the ratio effect of the approximation).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "pfpl_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liborcpfpl.so")

F32, F64 = 0, 1
ABS, REL, NOA = 0, 1, 2
FLAG_RAWWORDS, FLAG_MS = 1, 2
OK, ERR_ARG, ERR_BOUND, ERR_CAPACITY, ERR_CORRUPT = 0, -1, -2, -3, -4
CHUNK_BYTES = 16384
HEADER_BYTES = 48

_BOUNDS = {"abs": ABS, "rel": REL, "noa": NOA}


def build(force: bool = False) -> str:
    """Compile the oracle with IEEE-strict flags (no FMA contraction)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-ffp-contract=off",
               "-fno-fast-math", "-fopenmp", "-Wall", "-Wno-unused-function",
               _SRC, "-o", _LIB_PATH + ".tmp", "-lm"]
        subprocess.run(cmd, check=True)
        os.replace(_LIB_PATH + ".tmp", _LIB_PATH)
    return _LIB_PATH


class _Params(ctypes.Structure):
    _fields_ = [
        ("dtype", ctypes.c_int), ("bound", ctypes.c_int), ("flags", ctypes.c_int),
        ("eps", ctypes.c_double), ("range", ctypes.c_double),
        ("eps_eff_f", ctypes.c_float), ("inv_f", ctypes.c_float), ("eb2_f", ctypes.c_float),
        ("eps_eff_d", ctypes.c_double), ("inv_d", ctypes.c_double), ("eb2_d", ctypes.c_double),
        ("c_lo_f", ctypes.c_float), ("w_f", ctypes.c_float), ("inv_w_f", ctypes.c_float),
        ("c_lo_d", ctypes.c_double), ("w_d", ctypes.c_double), ("inv_w_d", ctypes.c_double),
        ("qconst", ctypes.c_uint64),
    ]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        vp, u64, i64 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int64
        L.orc_params_init.argtypes = [ctypes.POINTER(_Params), vp, u64, ctypes.c_int,
                                      ctypes.c_int, ctypes.c_double, ctypes.c_int]
        L.orc_params_init.restype = ctypes.c_int
        for nm, t in (("orc_log2p_f32", ctypes.c_float), ("orc_pow2p_f32", ctypes.c_float),
                      ("orc_log2p_f64", ctypes.c_double), ("orc_pow2p_f64", ctypes.c_double)):
            getattr(L, nm).argtypes = [t]
            getattr(L, nm).restype = t
        L.orc_quantize.argtypes = [ctypes.POINTER(_Params), vp, u64, vp]
        L.orc_quantize.restype = None
        L.orc_dequantize.argtypes = [ctypes.POINTER(_Params), vp, u64, vp]
        L.orc_dequantize.restype = None
        L.orc_delta_encode.argtypes = [vp, vp, ctypes.c_size_t, ctypes.c_int, ctypes.c_int]
        L.orc_delta_decode.argtypes = [vp, vp, ctypes.c_size_t, ctypes.c_int, ctypes.c_int]
        L.orc_shuffle.argtypes = [vp, ctypes.c_size_t, ctypes.c_int, vp]
        L.orc_unshuffle.argtypes = [vp, ctypes.c_size_t, ctypes.c_int, vp]
        L.orc_rze_encode.argtypes = [vp, vp]
        L.orc_rze_encode.restype = ctypes.c_size_t
        L.orc_rze_decode.argtypes = [vp, ctypes.c_size_t, vp]
        L.orc_rze_decode.restype = ctypes.c_long
        L.orc_max_compressed_bytes.argtypes = [u64, ctypes.c_int]
        L.orc_max_compressed_bytes.restype = u64
        L.orc_compress.argtypes = [vp, u64, ctypes.c_int, ctypes.c_int, ctypes.c_double,
                                   ctypes.c_int, vp, u64, ctypes.c_int]
        L.orc_compress.restype = i64
        L.orc_decompress.argtypes = [vp, u64, vp, u64, ctypes.POINTER(u64), ctypes.c_int]
        L.orc_decompress.restype = ctypes.c_int
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _dtype_code(x: np.ndarray) -> int:
    if x.dtype == np.float32:
        return F32
    if x.dtype == np.float64:
        return F64
    raise TypeError(f"unsupported dtype {x.dtype}")


def _bound_code(bound) -> int:
    return _BOUNDS[bound] if isinstance(bound, str) else int(bound)


class OracleError(RuntimeError):
    def __init__(self, code: int):
        super().__init__(f"oracle error {code}")
        self.code = code


def params(x: np.ndarray, bound, eps: float, ms: bool = False) -> _Params:
    x = np.ascontiguousarray(x)
    P = _Params()
    st = lib().orc_params_init(ctypes.byref(P), _ptr(x), x.size, _dtype_code(x),
                               _bound_code(bound), float(eps), int(ms))
    if st != OK:
        raise OracleError(st)
    return P


def quantize(x: np.ndarray, bound, eps: float, P: _Params | None = None) -> np.ndarray:
    x = np.ascontiguousarray(x)
    P = P or params(x, bound, eps)
    q = np.empty(x.size, dtype=np.uint32 if x.dtype == np.float32 else np.uint64)
    lib().orc_quantize(ctypes.byref(P), _ptr(x), x.size, _ptr(q))
    return q


def dequantize(q: np.ndarray, P: _Params) -> np.ndarray:
    q = np.ascontiguousarray(q)
    out = np.empty(q.size, dtype=np.float32 if q.dtype == np.uint32 else np.float64)
    lib().orc_dequantize(ctypes.byref(P), _ptr(q), q.size, _ptr(out))
    return out


def delta_encode(q: np.ndarray, bits: int, ms: bool = False) -> np.ndarray:
    q = np.ascontiguousarray(q, dtype=np.uint64)
    r = np.empty_like(q)
    lib().orc_delta_encode(_ptr(q), _ptr(r), q.size, bits, int(ms))
    return r


def delta_decode(r: np.ndarray, bits: int, ms: bool = False) -> np.ndarray:
    r = np.ascontiguousarray(r, dtype=np.uint64)
    q = np.empty_like(r)
    lib().orc_delta_decode(_ptr(r), _ptr(q), r.size, bits, int(ms))
    return q


def shuffle(r: np.ndarray, bits: int) -> np.ndarray:
    r = np.ascontiguousarray(r, dtype=np.uint64)
    S = np.empty(r.size * bits // 8, dtype=np.uint8)
    lib().orc_shuffle(_ptr(r), r.size, bits, _ptr(S))
    return S


def unshuffle(S: np.ndarray, cw: int, bits: int) -> np.ndarray:
    S = np.ascontiguousarray(S, dtype=np.uint8)
    r = np.empty(cw, dtype=np.uint64)
    lib().orc_unshuffle(_ptr(S), cw, bits, _ptr(r))
    return r


def rze_encode(X1: np.ndarray) -> bytes:
    X1 = np.ascontiguousarray(X1, dtype=np.uint8)
    assert X1.size == 16384
    out = np.empty(4 + 32 + 256 + 2048 + 16384, dtype=np.uint8)
    n = lib().orc_rze_encode(_ptr(X1), _ptr(out))
    return out[:n].tobytes()


def rze_decode(buf: bytes):
    a = np.frombuffer(buf, dtype=np.uint8).copy() if len(buf) else np.zeros(1, np.uint8)
    X1 = np.empty(16384, dtype=np.uint8)
    k = lib().orc_rze_decode(_ptr(a), len(buf), _ptr(X1))
    return (None, k) if k < 0 else (X1, k)


def log2p_f32(a: float) -> float:
    return lib().orc_log2p_f32(float(a))


def pow2p_f32(y: float) -> float:
    return lib().orc_pow2p_f32(float(y))


def log2p_f64(a: float) -> float:
    return lib().orc_log2p_f64(float(a))


def pow2p_f64(y: float) -> float:
    return lib().orc_pow2p_f64(float(y))


def max_compressed_bytes(n: int, dtype) -> int:
    code = dtype if isinstance(dtype, int) else (F32 if np.dtype(dtype) == np.float32 else F64)
    return int(lib().orc_max_compressed_bytes(n, code))


def compress(x: np.ndarray, bound, eps: float, ms: bool = False, nthreads: int = 1) -> bytes:
    """Whole-stream compression (O0-O7). Returns the stream bytes."""
    x = np.ascontiguousarray(x)
    dt = _dtype_code(x)
    cap = max_compressed_bytes(x.size, dt)
    out = np.empty(cap, dtype=np.uint8)
    n = lib().orc_compress(_ptr(x), x.size, dt, _bound_code(bound), float(eps), int(ms),
                           _ptr(out), cap, int(nthreads))
    if n < 0:
        raise OracleError(int(n))
    return out[:n].tobytes()


def decompress(buf: bytes, nthreads: int = 1) -> np.ndarray:
    """Whole-stream decompression (O8)."""
    a = np.frombuffer(buf, dtype=np.uint8)
    if len(a) < HEADER_BYTES:
        raise OracleError(ERR_CORRUPT)
    dt = a[5]
    n = int.from_bytes(bytes(a[8:16]), "little")
    if dt not in (F32, F64) or n > (1 << 40):
        raise OracleError(ERR_CORRUPT)
    out = np.empty(n, dtype=np.float32 if dt == F32 else np.float64)
    nout = ctypes.c_uint64(0)
    st = lib().orc_decompress(_ptr(a), len(a), _ptr(out), out.nbytes, ctypes.byref(nout),
                              int(nthreads))
    if st != OK:
        raise OracleError(st)
    return out
