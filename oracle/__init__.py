"""ctypes wrapper around the plain C++ oracle (oracle/lcf_oracle.cpp).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this package. The product path
(paper_conf_asplos_azamifb25_b200) never imports it.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lcf_oracle.cpp")
_HDR = os.path.join(_HERE, "lcf_oracle.h")
_LIB = os.path.join(_HERE, "liblcf_oracle.so")

ALGOS = {"SPspeed": 0, "SPratio": 1, "DPspeed": 2, "DPratio": 3}
WORD_DTYPE = {0: np.uint32, 1: np.uint32, 2: np.uint64, 3: np.uint64}


class OracleError(RuntimeError):
    def __init__(self, status: int, what: str):
        super().__init__(f"{what}: oracle status {status}")
        self.status = status


def build(force: bool = False) -> str:
    """Compile the oracle with plain g++ -O2 (no SIMD intrinsics, no -march)."""
    newest = max(os.path.getmtime(_SRC), os.path.getmtime(_HDR))
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < newest:
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC",
                               "-Wall", "-Wextra", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        sz, i32, u64 = ctypes.c_size_t, ctypes.c_int, ctypes.c_uint64
        vp = ctypes.c_void_p
        L.lcfo_max_compressed_size.argtypes = [i32, sz]
        L.lcfo_max_compressed_size.restype = sz
        for f in ("lcfo_compress", "lcfo_decompress"):
            getattr(L, f).argtypes = [i32, vp, sz, vp, sz, ctypes.POINTER(sz)]
            getattr(L, f).restype = i32
        L.lcfo_compress_chunks.argtypes = [i32, vp, sz, u64, u64, vp, vp, sz, ctypes.POINTER(u64)]
        L.lcfo_compress_chunks.restype = i32
        for f in ("lcfo_diffms32_enc", "lcfo_diffms32_dec", "lcfo_diffms64_enc",
                  "lcfo_diffms64_dec", "lcfo_bit32_enc", "lcfo_bit32_dec"):
            getattr(L, f).argtypes = [vp, sz, vp]
            getattr(L, f).restype = None
        for f in ("lcfo_mplg32_enc", "lcfo_mplg64_enc", "lcfo_rze_enc", "lcfo_raze_enc", "lcfo_rare_enc"):
            getattr(L, f).argtypes = [vp, sz, vp]
            getattr(L, f).restype = sz
        for f in ("lcfo_mplg32_dec", "lcfo_mplg64_dec", "lcfo_rze_dec"):
            getattr(L, f).argtypes = [vp, sz, sz, vp]
            getattr(L, f).restype = i32
        for f in ("lcfo_raze_dec", "lcfo_rare_dec"):
            getattr(L, f).argtypes = [vp, sz, vp, sz, ctypes.POINTER(sz)]
            getattr(L, f).restype = i32
        L.lcfo_fcm_hash.argtypes = [vp, sz, vp]
        L.lcfo_fcm_hash.restype = None
        L.lcfo_fcm_match.argtypes = [vp, vp, sz, vp, vp]
        L.lcfo_fcm_match.restype = None
        L.lcfo_fcm_dec.argtypes = [vp, vp, sz, vp]
        L.lcfo_fcm_dec.restype = i32
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _algo(a) -> int:
    return ALGOS[a] if isinstance(a, str) else int(a)


def _as_bytes(a) -> np.ndarray:
    if isinstance(a, (bytes, bytearray, memoryview)):
        return np.frombuffer(bytes(a), dtype=np.uint8)
    return np.ascontiguousarray(a).view(np.uint8).reshape(-1)


# ---- whole streams ---------------------------------------------------------

def max_compressed_size(algo, in_bytes: int) -> int:
    return int(lib().lcfo_max_compressed_size(_algo(algo), in_bytes))


def compress(algo, data) -> bytes:
    """Compress an array (its raw bytes) into an LCF1 stream (FORMAT.md)."""
    a = _algo(algo)
    src = _as_bytes(data)
    cap = max(max_compressed_size(a, src.size), 32)
    out = np.zeros(cap, dtype=np.uint8)
    nb = ctypes.c_size_t(0)
    st = lib().lcfo_compress(a, _ptr(src), src.size, _ptr(out), cap, ctypes.byref(nb))
    if st:
        raise OracleError(st, "compress")
    return out[: nb.value].tobytes()


def decompress(algo, stream, out_capacity: int | None = None) -> np.ndarray:
    """Decompress to the word array (uint32 / uint64 view of the floats)."""
    a = _algo(algo)
    src = _as_bytes(stream)
    if out_capacity is None:
        out_capacity = int.from_bytes(src[8:16].tobytes(), "little") if src.size >= 16 else 0
    out = np.zeros(max(out_capacity, 1), dtype=np.uint8)
    nb = ctypes.c_size_t(0)
    st = lib().lcfo_decompress(a, _ptr(src), src.size, _ptr(out), out_capacity, ctypes.byref(nb))
    if st:
        raise OracleError(st, "decompress")
    return out[: nb.value].view(WORD_DTYPE[a]).copy()


def decompress_status(algo, stream, out_capacity: int | None = None) -> int:
    try:
        decompress(algo, stream, out_capacity)
        return 0
    except OracleError as e:
        return e.status


def compress_chunks(algo, data, first_chunk: int, n_chunks: int):
    """Size-table slice and padded payload piece for a chunk range."""
    a = _algo(algo)
    src = _as_bytes(data)
    table = np.zeros(max(n_chunks, 1), dtype=np.uint32)
    cap = n_chunks * 16400 + 16
    payload = np.zeros(cap, dtype=np.uint8)
    pb = ctypes.c_uint64(0)
    st = lib().lcfo_compress_chunks(a, _ptr(src), src.size, first_chunk, n_chunks,
                                    _ptr(table), _ptr(payload), cap, ctypes.byref(pb))
    if st:
        raise OracleError(st, "compress_chunks")
    return table[:n_chunks].copy(), payload[: pb.value].tobytes()


# ---- stages ----------------------------------------------------------------

def diffms_enc(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x)
    u = np.empty_like(x)
    f = lib().lcfo_diffms32_enc if x.dtype == np.uint32 else lib().lcfo_diffms64_enc
    f(_ptr(x), x.size, _ptr(u))
    return u


def diffms_dec(u: np.ndarray) -> np.ndarray:
    u = np.ascontiguousarray(u)
    x = np.empty_like(u)
    f = lib().lcfo_diffms32_dec if u.dtype == np.uint32 else lib().lcfo_diffms64_dec
    f(_ptr(u), u.size, _ptr(x))
    return x


def mplg_enc(u: np.ndarray) -> bytes:
    u = np.ascontiguousarray(u)
    out = np.zeros(u.nbytes + 64, dtype=np.uint8)
    f = lib().lcfo_mplg32_enc if u.dtype == np.uint32 else lib().lcfo_mplg64_enc
    n = f(_ptr(u), u.size, _ptr(out))
    return out[:n].tobytes()


def mplg_dec(b: bytes, n: int, dtype) -> np.ndarray:
    src = _as_bytes(b)
    u = np.zeros(n, dtype=dtype)
    f = lib().lcfo_mplg32_dec if np.dtype(dtype) == np.uint32 else lib().lcfo_mplg64_dec
    st = f(_ptr(src), src.size, n, _ptr(u))
    if st:
        raise OracleError(st, "mplg_dec")
    return u


def bit32_enc(u: np.ndarray) -> np.ndarray:
    u = np.ascontiguousarray(u, dtype=np.uint32)
    t = np.empty_like(u)
    lib().lcfo_bit32_enc(_ptr(u), u.size, _ptr(t))
    return t


def bit32_dec(t: np.ndarray) -> np.ndarray:
    t = np.ascontiguousarray(t, dtype=np.uint32)
    u = np.empty_like(t)
    lib().lcfo_bit32_dec(_ptr(t), t.size, _ptr(u))
    return u


def rze_enc(d) -> bytes:
    src = _as_bytes(d)
    out = np.zeros(src.size + src.size // 4 + 16, dtype=np.uint8)
    n = lib().lcfo_rze_enc(_ptr(src), src.size, _ptr(out))
    return out[:n].tobytes()


def rze_dec(b: bytes, L: int) -> bytes:
    src = _as_bytes(b)
    out = np.zeros(max(L, 1), dtype=np.uint8)
    st = lib().lcfo_rze_dec(_ptr(src), src.size, L, _ptr(out))
    if st:
        raise OracleError(st, "rze_dec")
    return out[:L].tobytes()


def fcm_hash(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.uint64)
    h = np.empty(x.size, dtype=np.uint32)
    lib().lcfo_fcm_hash(_ptr(x), x.size, _ptr(h))
    return h


def fcm_match(x: np.ndarray, h: np.ndarray):
    x = np.ascontiguousarray(x, dtype=np.uint64)
    h = np.ascontiguousarray(h, dtype=np.uint32)
    V = np.empty_like(x)
    D = np.empty_like(x)
    lib().lcfo_fcm_match(_ptr(x), _ptr(h), x.size, _ptr(V), _ptr(D))
    return V, D


def fcm_dec(V: np.ndarray, D: np.ndarray) -> np.ndarray:
    V = np.ascontiguousarray(V, dtype=np.uint64)
    D = np.ascontiguousarray(D, dtype=np.uint64)
    x = np.empty_like(V)
    st = lib().lcfo_fcm_dec(_ptr(V), _ptr(D), V.size, _ptr(x))
    if st:
        raise OracleError(st, "fcm_dec")
    return x


def _adaptive_enc(f, d) -> bytes:
    src = _as_bytes(d)
    out = np.zeros(src.size + 8, dtype=np.uint8)
    n = f(_ptr(src), src.size, _ptr(out))
    return out[:n].tobytes()


def _adaptive_dec(f, b, what) -> bytes:
    src = _as_bytes(b)
    out = np.zeros(70000, dtype=np.uint8)
    L = ctypes.c_size_t(0)
    st = f(_ptr(src), src.size, _ptr(out), out.size, ctypes.byref(L))
    if st:
        raise OracleError(st, what)
    return out[: L.value].tobytes()


def raze_enc(d) -> bytes:
    return _adaptive_enc(lib().lcfo_raze_enc, d)


def rare_enc(d) -> bytes:
    return _adaptive_enc(lib().lcfo_rare_enc, d)


def raze_dec(b) -> bytes:
    return _adaptive_dec(lib().lcfo_raze_dec, b, "raze_dec")


def rare_dec(b) -> bytes:
    return _adaptive_dec(lib().lcfo_rare_dec, b, "rare_dec")
