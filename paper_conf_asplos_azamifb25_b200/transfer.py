"""Compressed point-to-point transfer.

The paper's motivation: a compressor pays off on a link when it
runs faster than link speed × ratio. NVLink 5 moves 900 GB/s per direction;
SPspeed/DPspeed compress at 2.3 TB/s and decompress at 2.4–2.8 TB/s on B200
(DESIGN.md §10). A stream of compression ratio R therefore crosses the link
at up to min(compress, 0.9·R TB/s, decompress) of uncompressed bytes.

Protocol (one sender, one receiver, any torch.distributed backend):
  preamble  int64[4]  magic, algo, n_bytes, slice_bytes
  per slice uint8[32] the slice's LCF1 sub-stream header (FORMAT.md §1)
            uint8[L]  the rest of the sub-stream: size table slice and payload,
                      L = round16(32 + 4·chunks) − 32 + payload_bytes
The input is cut into slices of whole 16 KiB chunks. Chunk encodings are
context-free (L104), so every slice is a self-contained LCF1 stream whose
chunks are exactly those of the whole array's stream (the stitched sequence of
sub-streams carries the same table entries and payload bytes as lcf_compress
of the whole array). The sender compresses slice i+1 while slice i is on the
wire (NCCL runs on its own stream, ordered after the compress by torch); the
receiver posts the next header receive before decoding slice i. DPratio is not
chunk-local (FCM spans the array, L170): it travels as one stream.

`codec` selects the slice coder: the B200 library (`lcf`, CUDA tensors, NCCL)
or the CPU codec (`lcf_cpu`, CPU tensors, e.g. gloo in the multi-process CPU
tests). The protocol code is the same for both.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np
import torch
import torch.distributed as dist

from .lcf import ALGOS

MAGIC = 0x4C434654  # "TFCL"
CHUNK = 16384
HEADER = 32


def _algo_id(algo) -> int:
    return ALGOS[algo] if isinstance(algo, str) else int(algo)


def _word_dtype(a: int):
    return torch.int32 if a in (0, 1) else torch.int64


def round16(v: int) -> int:
    return (v + 15) & ~15


def substream_bytes(header: np.ndarray) -> int:
    """Length of an LCF1 (sub-)stream from its 32-byte header."""
    h = np.frombuffer(np.ascontiguousarray(header).tobytes(), np.uint64)
    n_chunks, payload = int(h[2]), int(h[3])
    return round16(HEADER + 4 * n_chunks) + payload


class GpuCodec:
    """Slices through the B200 library (CUDA tensors)."""

    def __init__(self):
        from . import lcf
        self.lcf = lcf

    def compress(self, a: int, words: torch.Tensor) -> torch.Tensor:
        return self.lcf.compress(a, words)  # synchronising: the size is needed to post the send

    def decompress_into(self, a: int, sub: torch.Tensor, out_words: torch.Tensor) -> None:
        self.lcf.lcf_decompress(a, None, sub, sub.numel(), out_words, out_words.numel() * out_words.element_size(),
                                sync=False)

    def finish(self) -> None:
        self.lcf.lcf_check_stream()  # any malformed slice → LcfError (CORRUPT_STREAM)


class CpuCodec:
    """Slices through the multi-threaded CPU codec (CPU tensors)."""

    def __init__(self, n_threads: int = 0):
        from . import lcf_cpu
        self.cpu = lcf_cpu
        self.n_threads = n_threads

    def compress(self, a: int, words: torch.Tensor) -> torch.Tensor:
        return torch.from_numpy(self.cpu.lcf_cpu_compress(a, words.numpy(), self.n_threads).copy())

    def decompress_into(self, a: int, sub: torch.Tensor, out_words: torch.Tensor) -> None:
        w = self.cpu.lcf_cpu_decompress(a, sub.numpy(), out_words.numel() * out_words.element_size(), self.n_threads)
        out_words.copy_(torch.from_numpy(w.view(out_words.numpy().dtype)))

    def finish(self) -> None:
        pass


@dataclass
class TransferStats:
    n_bytes: int
    wire_bytes: int
    slices: int

    @property
    def ratio(self) -> float:
        return self.n_bytes / max(1, self.wire_bytes)


def _whole(n_bytes: int) -> int:
    """A slice size that covers n_bytes in one slice."""
    return max(CHUNK, (n_bytes + CHUNK - 1) // CHUNK * CHUNK)


def _slices(n_bytes: int, word_bytes: int, slice_bytes: int):
    step = max(CHUNK, slice_bytes // CHUNK * CHUNK)
    off = 0
    while off < n_bytes:
        end = min(n_bytes, off + step)
        yield off // word_bytes, end // word_bytes
        off = end


def send_compressed(x: torch.Tensor, dst: int, algo, codec=None, group=None,
                    slice_bytes: int = 64 << 20) -> TransferStats:
    """Send the words of `x` (int32 view for SP codecs, int64 for DP) to rank
    `dst` as compressed sub-streams; returns the byte counts."""
    a = _algo_id(algo)
    codec = codec or (GpuCodec() if x.is_cuda else CpuCodec())
    words = x.reshape(-1).view(_word_dtype(a))
    wb = words.element_size()
    n_bytes = words.numel() * wb
    if a == 3:  # DPratio: one stream (FCM spans the array)
        slice_bytes = _whole(n_bytes)
    pre = torch.tensor([MAGIC, a, n_bytes, slice_bytes], dtype=torch.int64, device=x.device)
    dist.send(pre, dst, group=group)
    wire, k, pending = 0, 0, []
    for w0, w1 in _slices(n_bytes, wb, slice_bytes):
        sub = codec.compress(a, words[w0:w1])  # overlaps the previous slice's sends
        parts = (sub[:HEADER].contiguous(), sub[HEADER:].contiguous())
        pending.append((parts, [dist.isend(t, dst, group=group) for t in parts]))
        wire += sub.numel()
        k += 1
        if len(pending) > 2:  # ≤ 2 slices in flight; their buffers stay referenced until sent
            for r in pending.pop(0)[1]:
                r.wait()
    for _, reqs in pending:
        for r in reqs:
            r.wait()
    return TransferStats(n_bytes, wire, k)


def substreams(words: torch.Tensor, algo, codec=None, slice_bytes: int = 64 << 20):
    """The sub-streams `send_compressed` puts on the wire, in order (for checks
    and for a caller that stores or forwards them)."""
    a = _algo_id(algo)
    codec = codec or (GpuCodec() if words.is_cuda else CpuCodec())
    w = words.reshape(-1).view(_word_dtype(a))
    n_bytes = w.numel() * w.element_size()
    if a == 3:
        slice_bytes = _whole(n_bytes)
    return [codec.compress(a, w[w0:w1]) for w0, w1 in _slices(n_bytes, w.element_size(), slice_bytes)]


def recv_compressed(src: int, algo, device=None, codec=None, group=None, out: torch.Tensor | None = None):
    """Receive an array sent by `send_compressed`; returns (words, stats). The
    words are int32 (SP codecs) or int64 (DP codecs); view them as float32 /
    float64."""
    a = _algo_id(algo)
    device = torch.device(device) if device is not None else (out.device if out is not None else torch.device("cpu"))
    codec = codec or (GpuCodec() if device.type == "cuda" else CpuCodec())
    pre = torch.empty(4, dtype=torch.int64, device=device)
    dist.recv(pre, src, group=group)
    magic, sa, n_bytes, slice_bytes = (int(v) for v in pre.cpu().tolist())
    if magic != MAGIC or sa != a:
        raise ValueError(f"recv_compressed: bad preamble (magic {magic:#x}, algo {sa} vs {a})")
    wdt = _word_dtype(a)
    wb = 4 if wdt == torch.int32 else 8
    if out is None:
        out = torch.empty(n_bytes // wb, dtype=wdt, device=device)
    words = out.reshape(-1).view(wdt)
    if words.numel() * wb != n_bytes:
        raise ValueError("recv_compressed: output size does not match the sender's array")
    wire, k = 0, 0
    bounds = list(_slices(n_bytes, wb, slice_bytes))
    hdr = torch.empty(HEADER, dtype=torch.uint8, device=device)
    req = dist.irecv(hdr, src, group=group) if bounds else None
    for i, (w0, w1) in enumerate(bounds):
        req.wait()
        L = substream_bytes(hdr.cpu().numpy())  # the slice's size: one 32-byte read
        sub = torch.empty(L, dtype=torch.uint8, device=device)
        sub[:HEADER].copy_(hdr)
        if L > HEADER:
            dist.recv(sub[HEADER:], src, group=group)
        if i + 1 < len(bounds):  # the next header is posted before this slice decodes
            hdr = torch.empty(HEADER, dtype=torch.uint8, device=device)
            req = dist.irecv(hdr, src, group=group)
        codec.decompress_into(a, sub, words[w0:w1])
        wire += L
        k += 1
    codec.finish()
    return out, TransferStats(n_bytes, wire, k)
