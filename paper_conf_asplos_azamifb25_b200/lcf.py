"""Thin ctypes binding of liblcf.so (include/lcf.h): same names, argument
marshalling only. Every step of the codec runs in the library's CUDA kernels;
there is no Python or CPU fallback — if liblcf.so is missing or no CUDA device
is usable, calls raise.

Device buffers are passed as torch CUDA tensors (or raw integer addresses);
streams as torch.cuda.Stream, raw handles, or None (= torch's current stream).
"""
from __future__ import annotations

import ctypes
import os

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("LCF_LIB_PATH") or os.path.join(PKG, "liblcf.so")

ALGOS = {"SPspeed": 0, "SPratio": 1, "DPspeed": 2, "DPratio": 3}
DTYPES = {"float32": 0, "float64": 1}
ALGO_DTYPE = {0: 0, 1: 0, 2: 1, 3: 1}
STATUS = {0: "SUCCESS", 1: "INVALID_ARGUMENT", 2: "DTYPE_MISMATCH", 3: "BUFFER_TOO_SMALL",
          4: "CORRUPT_STREAM", 5: "CUDA", 6: "OUT_OF_MEMORY"}


class LcfError(RuntimeError):
    def __init__(self, status: int, what: str):
        super().__init__(f"{what}: LCF_ERROR_{STATUS.get(status, status)}")
        self.status = status


_lib = None


class DpView(ctypes.Structure):
    """lcf_dp_view (include/lcf.h): one shard's decoded words and pending bitmap."""
    _fields_ = [("first_word", ctypes.c_uint64), ("n_words", ctypes.c_uint64), ("d_words", ctypes.c_void_p),
                ("d_pending", ctypes.c_void_p)]


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_asplos_azamifb25_b200.build` "
                              "or __graft_entry__.build() (no CPU fallback exists)")
        L = ctypes.CDLL(LIB_PATH)
        sz, u64, i32, vp = ctypes.c_size_t, ctypes.c_uint64, ctypes.c_int, ctypes.c_void_p
        psz = ctypes.POINTER(sz)
        L.lcf_max_compressed_size.argtypes = [i32, i32, sz]
        L.lcf_max_compressed_size.restype = sz
        L.lcf_num_chunks.argtypes = [i32, sz]
        L.lcf_num_chunks.restype = u64
        for f in ("lcf_compress", "lcf_decompress", "lcf_compress_host", "lcf_decompress_host"):
            getattr(L, f).argtypes = [i32, i32, vp, sz, vp, sz, psz, vp]
            getattr(L, f).restype = i32
        L.lcf_get_info.argtypes = [vp, sz, ctypes.POINTER(i32), ctypes.POINTER(i32), psz, psz, vp]
        L.lcf_get_info.restype = i32
        L.lcf_check_stream.argtypes = [vp]
        L.lcf_check_stream.restype = i32
        L.lcf_compress_shard.argtypes = [i32, i32, vp, sz, sz, u64, vp, vp, sz, vp, vp]
        L.lcf_compress_shard.restype = i32
        L.lcf_write_header.argtypes = [i32, i32, sz, u64, vp, vp]
        L.lcf_write_header.restype = i32
        L.lcf_dpratio_summary_bytes.argtypes = []
        L.lcf_dpratio_summary_bytes.restype = sz
        L.lcf_dpratio_shard_summary.argtypes = [vp, sz, sz, u64, vp, vp]
        L.lcf_dpratio_shard_summary.restype = i32
        L.lcf_dpratio_merge_summaries.argtypes = [vp, sz, vp, vp]
        L.lcf_dpratio_merge_summaries.restype = i32
        L.lcf_dpratio_compress_shard.argtypes = [vp, sz, sz, u64, vp, vp, vp, sz, vp, vp]
        L.lcf_dpratio_compress_shard.restype = i32
        L.lcf_dpratio_decompress_shard.argtypes = [vp, sz, u64, vp, sz, vp, vp]
        L.lcf_dpratio_decompress_shard.restype = i32
        L.lcf_dpratio_merge_summary_ptrs.argtypes = [ctypes.POINTER(vp), sz, vp, vp]
        L.lcf_dpratio_merge_summary_ptrs.restype = i32
        for f in ("lcf_dpratio_find_roots", "lcf_dpratio_gather_roots"):
            getattr(L, f).argtypes = [ctypes.POINTER(DpView), sz, sz, vp]
            getattr(L, f).restype = i32
        L.lcf_ipc_export.argtypes = [vp, ctypes.c_char_p, ctypes.POINTER(u64)]
        L.lcf_ipc_export.restype = i32
        L.lcf_ipc_import.argtypes = [ctypes.c_char_p, u64, ctypes.POINTER(vp)]
        L.lcf_ipc_import.restype = i32
        L.lcf_ipc_close.argtypes = [vp]
        L.lcf_ipc_close.restype = i32
        L.lcf_launch_count.argtypes = []
        L.lcf_launch_count.restype = u64
        L.lcf_profile_enable.argtypes = [i32]
        L.lcf_profile_enable.restype = None
        L.lcf_profile_report.argtypes = [ctypes.c_char_p, sz]
        L.lcf_profile_report.restype = sz
        _lib = L
    return _lib


def _algo(a) -> int:
    return ALGOS[a] if isinstance(a, str) else int(a)


def _dtype(d, algo=None) -> int:
    if d is None:
        return ALGO_DTYPE[algo]
    if isinstance(d, str):
        return DTYPES[d]
    try:
        import torch
        if d == torch.float32:
            return 0
        if d == torch.float64:
            return 1
    except ImportError:
        pass
    return int(d)


def _ptr(x):
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "ctypes"):  # numpy (host) array
        return x.ctypes.data
    raise TypeError(type(x))


def _stream(s):
    if s is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(s, int):
        return s
    return s.cuda_stream


def _check(st: int, what: str):
    if st:
        raise LcfError(st, what)


# ---- the C ABI, same names -----------------------------------------------------

def lcf_max_compressed_size(algo, dtype, in_bytes: int) -> int:
    a = _algo(algo)
    return int(lib().lcf_max_compressed_size(a, _dtype(dtype, a), in_bytes))


def lcf_num_chunks(algo, in_bytes: int) -> int:
    return int(lib().lcf_num_chunks(_algo(algo), in_bytes))


def lcf_compress(algo, dtype, d_in, in_bytes, d_out, out_capacity, sync=True, stream=None):
    a = _algo(algo)
    n = ctypes.c_size_t(0)
    st = lib().lcf_compress(a, _dtype(dtype, a), _ptr(d_in), in_bytes, _ptr(d_out), out_capacity,
                            ctypes.byref(n) if sync else None, _stream(stream))
    _check(st, "lcf_compress")
    return n.value if sync else None


def lcf_decompress(algo, dtype, d_in, in_bytes, d_out, out_capacity, sync=True, stream=None):
    a = _algo(algo)
    n = ctypes.c_size_t(0)
    st = lib().lcf_decompress(a, _dtype(dtype, a), _ptr(d_in), in_bytes, _ptr(d_out), out_capacity,
                              ctypes.byref(n) if sync else None, _stream(stream))
    _check(st, "lcf_decompress")
    return n.value if sync else None


def lcf_get_info(d_in, in_bytes, stream=None) -> dict:
    al, dt = ctypes.c_int(0), ctypes.c_int(0)
    ub, cb = ctypes.c_size_t(0), ctypes.c_size_t(0)
    st = lib().lcf_get_info(_ptr(d_in), in_bytes, ctypes.byref(al), ctypes.byref(dt), ctypes.byref(ub),
                            ctypes.byref(cb), _stream(stream))
    _check(st, "lcf_get_info")
    return {"algo": al.value, "dtype": dt.value, "uncompressed_bytes": ub.value, "compressed_bytes": cb.value}


def lcf_check_stream(stream=None) -> None:
    _check(lib().lcf_check_stream(_stream(stream)), "lcf_check_stream")


def lcf_compress_host(algo, dtype, h_in, in_bytes, h_out, out_capacity, stream=None) -> int:
    a = _algo(algo)
    n = ctypes.c_size_t(0)
    _check(lib().lcf_compress_host(a, _dtype(dtype, a), _ptr(h_in), in_bytes, _ptr(h_out), out_capacity,
                                   ctypes.byref(n), _stream(stream)), "lcf_compress_host")
    return n.value


def lcf_decompress_host(algo, dtype, h_in, in_bytes, h_out, out_capacity, stream=None) -> int:
    a = _algo(algo)
    n = ctypes.c_size_t(0)
    _check(lib().lcf_decompress_host(a, _dtype(dtype, a), _ptr(h_in), in_bytes, _ptr(h_out), out_capacity,
                                     ctypes.byref(n), _stream(stream)), "lcf_decompress_host")
    return n.value


def lcf_compress_shard(algo, dtype, d_in_shard, shard_bytes, total_in_bytes, first_chunk, d_table_slice,
                       d_payload, payload_capacity, d_payload_bytes, stream=None) -> None:
    a = _algo(algo)
    _check(lib().lcf_compress_shard(a, _dtype(dtype, a), _ptr(d_in_shard), shard_bytes, total_in_bytes,
                                    first_chunk, _ptr(d_table_slice), _ptr(d_payload), payload_capacity,
                                    _ptr(d_payload_bytes), _stream(stream)), "lcf_compress_shard")


def lcf_dpratio_summary_bytes() -> int:
    return int(lib().lcf_dpratio_summary_bytes())


def lcf_dpratio_shard_summary(d_x, shard_bytes, total_in_bytes, first_word, d_summary, stream=None) -> None:
    _check(lib().lcf_dpratio_shard_summary(_ptr(d_x), shard_bytes, total_in_bytes, first_word, _ptr(d_summary),
                                           _stream(stream)), "lcf_dpratio_shard_summary")


def lcf_dpratio_merge_summaries(d_summaries, count, d_carry, stream=None) -> None:
    _check(lib().lcf_dpratio_merge_summaries(_ptr(d_summaries), count, _ptr(d_carry), _stream(stream)),
           "lcf_dpratio_merge_summaries")


def lcf_dpratio_compress_shard(d_x, shard_bytes, total_in_bytes, first_word, d_carry, d_table_slice, d_payload,
                               payload_capacity, d_payload_bytes, stream=None) -> None:
    _check(lib().lcf_dpratio_compress_shard(_ptr(d_x), shard_bytes, total_in_bytes, first_word, _ptr(d_carry),
                                            _ptr(d_table_slice), _ptr(d_payload), payload_capacity,
                                            _ptr(d_payload_bytes), _stream(stream)), "lcf_dpratio_compress_shard")


def lcf_dpratio_decompress_shard(d_in, in_bytes, first_word, d_out, out_capacity, d_pending, stream=None) -> None:
    _check(lib().lcf_dpratio_decompress_shard(_ptr(d_in), in_bytes, first_word, _ptr(d_out), out_capacity,
                                              _ptr(d_pending), _stream(stream)), "lcf_dpratio_decompress_shard")


def lcf_dpratio_merge_summary_ptrs(d_summaries, count, d_carry, stream=None) -> None:
    """d_summaries: list of device pointers (tensors or ints), shard order."""
    arr = (ctypes.c_void_p * max(1, count))(*[_ptr(p) for p in d_summaries[:count]])
    _check(lib().lcf_dpratio_merge_summary_ptrs(arr, count, _ptr(d_carry), _stream(stream)),
           "lcf_dpratio_merge_summary_ptrs")


def _views(views):
    """views: list of (first_word, n_words, d_words, d_pending)."""
    arr = (DpView * len(views))()
    for q, (f, n, w, p) in enumerate(views):
        arr[q] = DpView(f, n, _ptr(w), _ptr(p))
    return arr


def lcf_dpratio_find_roots(views, self_index, stream=None) -> None:
    _check(lib().lcf_dpratio_find_roots(_views(views), len(views), self_index, _stream(stream)),
           "lcf_dpratio_find_roots")


def lcf_dpratio_gather_roots(views, self_index, stream=None) -> None:
    _check(lib().lcf_dpratio_gather_roots(_views(views), len(views), self_index, _stream(stream)),
           "lcf_dpratio_gather_roots")


def lcf_ipc_export(d_ptr):
    """(64-byte handle, offset) of the device allocation holding d_ptr."""
    h = ctypes.create_string_buffer(64)
    off = ctypes.c_uint64()
    _check(lib().lcf_ipc_export(_ptr(d_ptr), h, ctypes.byref(off)), "lcf_ipc_export")
    return h.raw, int(off.value)


def lcf_ipc_import(handle: bytes, offset: int) -> int:
    p = ctypes.c_void_p()
    _check(lib().lcf_ipc_import(handle, offset, ctypes.byref(p)), "lcf_ipc_import")
    return int(p.value)


def lcf_ipc_close(d_ptr: int) -> None:
    _check(lib().lcf_ipc_close(d_ptr), "lcf_ipc_close")


def lcf_write_header(algo, dtype, total_in_bytes, total_payload_bytes, d_stream, stream=None) -> None:
    a = _algo(algo)
    _check(lib().lcf_write_header(a, _dtype(dtype, a), total_in_bytes, total_payload_bytes, _ptr(d_stream),
                                  _stream(stream)), "lcf_write_header")


def lcf_launch_count() -> int:
    return int(lib().lcf_launch_count())


def lcf_profile_enable(enable: bool) -> None:
    lib().lcf_profile_enable(1 if enable else 0)


def lcf_profile_report() -> dict:
    """{kernel name: (launches, total ms)} since enabling; clears the record."""
    buf = ctypes.create_string_buffer(1 << 16)
    lib().lcf_profile_report(buf, len(buf))
    out = {}
    for line in buf.value.decode().splitlines():
        name, cnt, ms = line.split()
        out[name] = (int(cnt), float(ms))
    return out


# ---- tensor conveniences (allocation + the calls above) ------------------------

def compress(algo, x, out=None, stream=None):
    """Compress a CUDA tensor; returns the uint8 stream tensor (trimmed view)."""
    import torch
    a = _algo(algo)
    nbytes = x.numel() * x.element_size()
    cap = lcf_max_compressed_size(a, None, nbytes)
    if out is None:
        out = torch.empty(cap, dtype=torch.uint8, device=x.device)
    n = lcf_compress(a, None, x, nbytes, out, out.numel(), sync=True, stream=stream)
    return out[:n]


def decompress(algo, s, out=None, stream=None):
    """Decompress a uint8 CUDA stream tensor into a new word tensor."""
    import torch
    a = _algo(algo)
    info = lcf_get_info(s, s.numel(), stream=stream)
    wdt = torch.int32 if a < 2 else torch.int64
    if out is None:
        out = torch.empty(info["uncompressed_bytes"] // (4 if a < 2 else 8), dtype=wdt, device=s.device)
    lcf_decompress(a, None, s, s.numel(), out, out.numel() * out.element_size(), sync=True, stream=stream)
    return out
