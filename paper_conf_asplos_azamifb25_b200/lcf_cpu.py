"""ctypes binding of liblcf_cpu.so (include/lcf_cpu.h): the multi-threaded CPU
codec, bit-compatible with the B200 stream. Argument
marshalling only; a separate library that the GPU binding (lcf.py) never
calls. Buffers are numpy arrays / bytes (host memory)."""
from __future__ import annotations

import ctypes
import os

import numpy as np

from .lcf import ALGO_DTYPE, ALGOS, LcfError

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("LCF_CPU_LIB_PATH") or os.path.join(PKG, "liblcf_cpu.so")
_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_asplos_azamifb25_b200.build`")
        L = ctypes.CDLL(LIB_PATH)
        sz, i32, vp = ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p
        L.lcf_cpu_max_compressed_size.argtypes = [i32, i32, sz]
        L.lcf_cpu_max_compressed_size.restype = sz
        for f in ("lcf_cpu_compress", "lcf_cpu_decompress"):
            getattr(L, f).argtypes = [i32, i32, vp, sz, vp, sz, ctypes.POINTER(sz), i32]
            getattr(L, f).restype = i32
        _lib = L
    return _lib


def _algo(a) -> int:
    return ALGOS[a] if isinstance(a, str) else int(a)


def _buf(a):
    a = np.ascontiguousarray(np.frombuffer(a, np.uint8) if isinstance(a, (bytes, bytearray)) else a)
    return a, a.ctypes.data_as(ctypes.c_void_p), a.nbytes


def lcf_cpu_max_compressed_size(algo, in_bytes: int) -> int:
    a = _algo(algo)
    return lib().lcf_cpu_max_compressed_size(a, ALGO_DTYPE.get(a, 0), in_bytes)


def lcf_cpu_compress(algo, data, n_threads: int = 0, dtype=None) -> np.ndarray:
    """Compress the words of `data` (a numpy array); returns the stream as u8."""
    a = _algo(algo)
    d, p, n = _buf(data)
    out = np.empty(max(32, lcf_cpu_max_compressed_size(a, n)), np.uint8)
    got = ctypes.c_size_t(0)
    st = lib().lcf_cpu_compress(a, ALGO_DTYPE.get(a, 0) if dtype is None else dtype, p, n,
                                out.ctypes.data_as(ctypes.c_void_p), out.nbytes, ctypes.byref(got), n_threads)
    if st:
        raise LcfError(st, "lcf_cpu_compress")
    return out[: got.value]


def lcf_cpu_decompress(algo, stream, out_capacity: int | None = None, n_threads: int = 0, dtype=None) -> np.ndarray:
    """Decompress an LCF1 stream; returns the words (u32 for SP codecs, u64 for DP)."""
    a = _algo(algo)
    s, p, n = _buf(stream)
    if out_capacity is None:
        out_capacity = int(np.frombuffer(s[8:16].tobytes(), np.uint64)[0]) if n >= 32 else 0
    out = np.empty(max(out_capacity, 1), np.uint8)
    got = ctypes.c_size_t(0)
    st = lib().lcf_cpu_decompress(a, ALGO_DTYPE.get(a, 0) if dtype is None else dtype, p, n,
                                  out.ctypes.data_as(ctypes.c_void_p), out_capacity, ctypes.byref(got), n_threads)
    if st:
        raise LcfError(st, "lcf_cpu_decompress")
    return out[: got.value].view(np.uint32 if a in (0, 1) else np.uint64)
