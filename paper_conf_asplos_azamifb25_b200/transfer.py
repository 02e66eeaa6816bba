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


# ---- fused compress + transfer over peer memory ----------------------------------

class P2PChannel:
    """Compression fused with the NVLink transfer (NEXT-3, the one-kernel form):
    the receiver's stream buffer is mapped into the sender by CUDA IPC
    (lcf_ipc_export / lcf_ipc_import), and the sender's lcf_compress writes the
    stream straight into it — every chunk's TMA bulk store crosses NVLink as
    soon as its decoupled look-back resolves, so the transfer overlaps the
    compression chunk by chunk, and no copy or NCCL payload message follows.
    The receiver decompresses from its own memory once a one-word signal
    (stream-ordered after the compress on the sender) arrives.

    Both ranks construct the channel (collectively) for arrays of up to
    `max_bytes`; `send` / `recv` then move one array each; `close` unmaps. The
    buffer is reused: a send waits for the receiver's release of the previous
    stream (recv releases it once its decode is enqueued, unless asked not
    to — then `release()`). Any
    torch.distributed backend carries the handle and the signal (NCCL: CUDA
    tensors; gloo: CPU tensors after a device synchronisation)."""

    def __init__(self, src: int, dst: int, algo, max_bytes: int, group=None):
        from . import lcf
        self.lcf, self.src, self.dst, self.group = lcf, src, dst, group
        self.a = _algo_id(algo)
        self.cap = lcf.lcf_max_compressed_size(self.a, None, max_bytes)
        self.rank = dist.get_rank(group)
        self.gloo = dist.get_backend(group) == "gloo"
        self.peer = None
        self.sent = 0  # streams sent (sender): every one after the first waits for a release
        dev = torch.device("cuda", torch.cuda.current_device())
        self.dev = dev
        msg = torch.zeros(72, dtype=torch.uint8)
        if self.rank == dst:
            self.buf = torch.empty(self.cap, dtype=torch.uint8, device=dev)
            h, off = lcf.lcf_ipc_export(self.buf)
            msg[:64] = torch.frombuffer(bytearray(h), dtype=torch.uint8)
            msg[64:] = torch.tensor([off], dtype=torch.int64).view(torch.uint8)
            dist.send(self._wire(msg), src, group=group)
        elif self.rank == src:
            m = self._wire(msg)
            dist.recv(m, dst, group=group)
            m = m.cpu()
            self.peer = lcf.lcf_ipc_import(bytes(m[:64].numpy()), int(m[64:].view(torch.int64)[0]))

    def _wire(self, t):
        return t if self.gloo else t.to(self.dev)

    def _signal(self, send: bool, value: int = 0, to=None, frm=None) -> int:
        t = self._wire(torch.tensor([value], dtype=torch.int64))
        if send:
            if self.gloo:
                torch.cuda.synchronize()  # the kernels before it (and their peer stores) are complete
            dist.send(t, self.dst if to is None else to, group=self.group)  # NCCL: stream-ordered
            return value
        dist.recv(t, self.src if frm is None else frm, group=self.group)
        return int(t.item())

    def send(self, x: torch.Tensor) -> int:
        """Compress x's words into the receiver's buffer; returns the stream
        bytes (read back from the local call, synchronising)."""
        words = x.reshape(-1).view(_word_dtype(self.a))
        nb = words.numel() * words.element_size()
        if self.sent:
            self._signal(False, frm=self.dst)  # the receiver has released the buffer
        n = self.lcf.lcf_compress(self.a, None, words, nb, self.peer, self.cap, sync=True)
        self._signal(True, n)
        self.sent += 1
        return n

    def recv(self, out: torch.Tensor, release: bool = True) -> int:
        """Decompress the array the sender wrote into this rank's buffer into
        `out` (its word view); returns the stream bytes."""
        n = self._signal(False)
        words = out.reshape(-1).view(_word_dtype(self.a))
        self.lcf.lcf_decompress(self.a, None, self.buf, n, words, words.numel() * words.element_size(), sync=False)
        if release:
            self.release()
        return n

    def release(self) -> None:
        """(receiver) the buffer may be overwritten by the next send."""
        self._signal(True, 0, to=self.src)

    def stream(self) -> torch.Tensor:
        """(receiver) the stream bytes of the last transfer, for checks."""
        return self.buf

    def close(self) -> None:
        """Both ranks: the sender takes the receiver's last release (each
        recv's release is matched here or by the next send), then unmaps."""
        if self.rank == self.src and self.sent:
            self._signal(False, frm=self.dst)
            self.sent = 0
        if self.peer is not None:
            self.lcf.lcf_ipc_close(self.peer)
            self.peer = None
