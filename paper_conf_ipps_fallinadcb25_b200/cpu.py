"""Multi-core CPU PFPL codec (libpfpl_cpu.so, include/pfpl_cpu.h).

The paper's OpenMP implementation for the host CPU of a B200 node.
Argument marshalling only (numpy arrays in host memory); every step runs in
paper_conf_ipps_fallinadcb25_b200/cpu/pfpl_cpu.c.  Streams are byte-identical
to the GPU library's.  This is a separate CPU product, not a fallback:
the GPU API never calls it.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

_lib = None
_BOUNDS = {"abs": 0, "rel": 1, "noa": 2}
_ERR = {-1: "invalid argument", -2: "invalid error bound", -3: "output capacity too small",
        -4: "corrupt stream"}


class PFPLCPUError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        super().__init__(f"pfpl_cpu error {code} ({_ERR.get(code, '?')}) {what}".strip())
        self.code = code


def lib():
    global _lib
    if _lib is None:
        path = _build.build_cpu()
        L = ctypes.CDLL(path)
        vp, u64, i32, dbl = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int, ctypes.c_double
        pu64 = ctypes.POINTER(ctypes.c_uint64)
        L.pfpl_cpu_max_compressed_bytes.argtypes = [u64, i32]
        L.pfpl_cpu_max_compressed_bytes.restype = u64
        L.pfpl_cpu_compress.argtypes = [vp, u64, i32, i32, dbl, ctypes.c_uint, vp, pu64, i32]
        L.pfpl_cpu_compress.restype = i32
        L.pfpl_cpu_decompress.argtypes = [vp, u64, vp, pu64, i32]
        L.pfpl_cpu_decompress.restype = i32
        L.pfpl_cpu_max_threads.argtypes = []
        L.pfpl_cpu_max_threads.restype = i32
        _lib = L
    return _lib


def max_threads() -> int:
    return int(lib().pfpl_cpu_max_threads())


def compress(x: np.ndarray, bound="abs", eps: float = 1e-3, ms: bool = False, nthreads: int = 0,
             out: np.ndarray | None = None):
    """Returns the stream as bytes, or, when a uint8 `out` buffer is given (reused
    across calls: no page faults on a fresh allocation), a view of it."""
    x = np.ascontiguousarray(x)
    if x.dtype not in (np.float32, np.float64):
        raise TypeError(f"PFPL compresses float32/float64, got {x.dtype}")
    dt = 0 if x.dtype == np.float32 else 1
    cap = int(lib().pfpl_cpu_max_compressed_bytes(x.size, dt))
    view = out is not None
    if out is None:
        out = np.empty(max(cap, 1), np.uint8)
    cap = out.size
    nb = ctypes.c_uint64(cap)
    st = lib().pfpl_cpu_compress(x.ctypes.data_as(ctypes.c_void_p), x.size, dt,
                                 _BOUNDS[bound] if isinstance(bound, str) else int(bound), float(eps),
                                 2 if ms else 0, out.ctypes.data_as(ctypes.c_void_p), ctypes.byref(nb),
                                 int(nthreads))
    if st:
        raise PFPLCPUError(st, "compress")
    return out[:nb.value] if view else out[:nb.value].tobytes()


def decompress(buf, nthreads: int = 0, out: np.ndarray | None = None) -> np.ndarray:
    a = np.frombuffer(buf, np.uint8) if not isinstance(buf, np.ndarray) else buf
    if a.size < 48:
        raise PFPLCPUError(-4, "stream shorter than its header")
    dt = int(a[5])
    n = int.from_bytes(bytes(a[8:16]), "little")
    if dt not in (0, 1) or n > (1 << 40):
        raise PFPLCPUError(-4, "header")
    if out is None:
        out = np.empty(max(n, 1), np.float32 if dt == 0 else np.float64)
    ob = ctypes.c_uint64(out.nbytes)
    st = lib().pfpl_cpu_decompress(a.ctypes.data_as(ctypes.c_void_p), a.size,
                                   out.ctypes.data_as(ctypes.c_void_p), ctypes.byref(ob), int(nthreads))
    if st:
        raise PFPLCPUError(st, "decompress")
    return out[:n]
