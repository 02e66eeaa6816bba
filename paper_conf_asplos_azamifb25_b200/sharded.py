"""Multi-GPU mode: one process per GPU, chunk-range shards of ONE stream
(BASELINE north_star "8-GPU mode").

Rank g owns chunks [⌊gC/G⌋, ⌊(g+1)C/G⌋) of the global input. It compresses its
shard into a *local* LCF1 stream. Chunks are context-free and shard boundaries
are chunk boundaries, so the local size table and payload ARE the global
stream's table slice and payload piece. The local payload byte count sits in
the local header at byte 24; it is all-gathered as a device u64 (NCCL over
NVLink/NVSwitch; gloo in the CPU tests) — the only exchange. An exclusive scan
over ranks gives each piece's offset, and rank 0 writes the global header. The
concatenation header ‖ table slices ‖ pad ‖ payload pieces is byte-identical to
the 1-GPU stream. Decompression needs no exchange: every rank decodes its local
stream.

DPratio shards by whole tiles with one more exchange (the FCM summaries, see
below); its pieces assemble into the 1-GPU stream the same way.
"""
from __future__ import annotations

from dataclasses import dataclass

HEADER = 32
CHUNK = 16384


def num_chunks(n_bytes: int) -> int:
    return -(-n_bytes // CHUNK)


def shard_chunks(n_bytes: int, world: int, rank: int):
    """(first_chunk, n_chunks) of `rank`'s contiguous chunk range."""
    C = num_chunks(n_bytes)
    first = C * rank // world
    last = C * (rank + 1) // world
    return first, last - first


def shard_bytes(n_bytes: int, world: int, rank: int):
    """(byte offset, byte length) of `rank`'s shard of the input."""
    first, k = shard_chunks(n_bytes, world, rank)
    start = first * CHUNK
    return start, max(0, min(n_bytes, (first + k) * CHUNK) - start)


def round16(v: int) -> int:
    return (v + 15) // 16 * 16


@dataclass
class Piece:
    """One rank's part of the global stream."""
    rank: int
    first_chunk: int
    n_chunks: int
    local_stream: object  # uint8 tensor: local header ‖ table slice ‖ pad ‖ payload
    payload_bytes: int
    payload_offset: int   # offset of this piece inside the global payload
    total_payload: int

    def table_slice(self):
        return self.local_stream[HEADER:HEADER + 4 * self.n_chunks]

    def payload(self):
        b = round16(HEADER + 4 * self.n_chunks)
        return self.local_stream[b:b + self.payload_bytes]


def exchange_counts(count_u64, group=None):
    """All-gather one u64 per rank (a 1-element int64 tensor on the process
    group's device) and return the list of counts — the single collective."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    out = torch.empty(world, dtype=torch.int64, device=count_u64.device)
    dist.all_gather_into_tensor(out, count_u64.reshape(1).to(torch.int64), group=group)
    return out


def compress_sharded(algo: str, shard, total_bytes: int, local_compress, group=None) -> Piece:
    """`shard` is this rank's slice of the global input (chunk-aligned);
    `local_compress(algo, shard) -> uint8 tensor` is the codec (lcf on GPU,
    the oracle in the CPU tests)."""
    import torch
    import torch.distributed as dist
    if algo == "DPratio":
        raise ValueError("DPratio runs whole fields per rank (FCM is a whole-array pass, L104)")
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    first, k = shard_chunks(total_bytes, world, rank)
    local = local_compress(algo, shard)
    count = local[24:32].view(torch.int64)  # local payload_bytes, left on its device
    counts = exchange_counts(count, group).cpu().tolist()
    offset = sum(counts[:rank])
    return Piece(rank, first, k, local, counts[rank], offset, sum(counts))


def global_header(algo: str, total_bytes: int, total_payload: int) -> bytes:
    """The 32-byte LCF1 header (FORMAT.md §1) for the assembled stream."""
    algo_id = {"SPspeed": 0, "SPratio": 1, "DPspeed": 2, "DPratio": 3}[algo]
    wb = 4 if algo.startswith("SP") else 8
    return (0x3146434C).to_bytes(4, "little") + bytes([1, algo_id, wb, 0]) + \
        total_bytes.to_bytes(8, "little") + num_chunks(total_bytes).to_bytes(8, "little") + \
        total_payload.to_bytes(8, "little")


def assemble(algo: str, total_bytes: int, pieces) -> bytes:
    """Concatenate gathered pieces (rank order) into the global stream bytes
    (identity tests only; outside any timed region)."""
    C = num_chunks(total_bytes)
    tables = b"".join(bytes(p.table_slice().cpu().numpy().tobytes()) for p in pieces)
    assert len(tables) == 4 * C
    base = round16(HEADER + 4 * C)
    pad = bytes(base - HEADER - 4 * C)
    payload = b"".join(bytes(p.payload().cpu().numpy().tobytes()) for p in pieces)
    total_payload = sum(p.payload_bytes for p in pieces)
    return global_header(algo, total_bytes, total_payload) + tables + pad + payload


def gather_pieces(piece: Piece, group=None):
    """Rank 0 receives every rank's Piece (object collective; tests only)."""
    import torch.distributed as dist
    payload = (piece.rank, piece.first_chunk, piece.n_chunks, piece.local_stream.cpu(), piece.payload_bytes,
               piece.payload_offset, piece.total_payload)
    out = [None] * dist.get_world_size(group)
    dist.all_gather_object(out, payload, group=group)
    return [Piece(*o) for o in out]


def lcf_local_compress(algo: str, shard):
    """GPU shard codec: lcf_compress into a local stream (device tensor)."""
    from . import lcf
    return lcf.compress(algo, shard)


def lcf_local_decompress(algo: str, local_stream, out=None):
    from . import lcf
    return lcf.decompress(algo, local_stream, out=out)


# ---- sharded DPratio -------------------------------------
# FCM (L170–185) compares a word with the ≤ 4 nearest preceding same-hash words
# anywhere before it. Ranks own whole 2048-word tiles; each computes a summary
# of its shard (per hash, its last ≤ 4 words), the summaries are all-gathered,
# and rank g merges those of ranks 0 … g−1 into its carry (lcf.h). With the
# carry, the shard's chunks are exactly the 1-GPU stream's chunks 2·t, 2·t+1 of
# its tiles t, and the pieces assemble like the chunk-local codecs'.

TILE_WORDS = 2048


def dp_shard_words(n_words: int, world: int, rank: int):
    """(first_word, n_words) of `rank`'s contiguous range of whole tiles."""
    T = -(-n_words // TILE_WORDS)
    t0, t1 = T * rank // world, T * (rank + 1) // world
    first = t0 * TILE_WORDS
    return first, max(0, min(n_words, t1 * TILE_WORDS) - first)


def dp_compress_piece(x_shard, n_total_words: int, first_word: int, carry, rank: int):
    """One shard's table slice, payload piece and device payload byte count
    (lcf_dpratio_compress_shard). x_shard: int64 CUDA tensor view of the
    shard's words inside a buffer that also holds the 3 words before it."""
    import torch
    from . import lcf
    nb = x_shard.numel() * 8
    tiles = -(-x_shard.numel() // TILE_WORDS)
    cap = max(16, 2 * tiles * CHUNK)
    table = torch.empty(max(1, 2 * tiles), dtype=torch.int32, device=x_shard.device)
    payload = torch.empty(cap, dtype=torch.uint8, device=x_shard.device)
    count = torch.zeros(1, dtype=torch.int64, device=x_shard.device)
    lcf.lcf_dpratio_compress_shard(x_shard, nb, 8 * n_total_words, first_word, carry, table, payload, cap, count)
    return table[:2 * tiles], payload, count


def dp_simulate_shards(x, world: int) -> bytes:
    """All ranks' steps on one device, in rank order (a summary pointer is a
    plain device pointer here): the assembled stream, for identity tests."""
    import torch
    from . import lcf
    n = x.numel()
    sb = lcf.lcf_dpratio_summary_bytes()
    sums = [torch.empty(sb, dtype=torch.uint8, device=x.device) for _ in range(world)]
    ranges = [dp_shard_words(n, world, g) for g in range(world)]
    for g, (f, k) in enumerate(ranges):
        lcf.lcf_dpratio_shard_summary(x[f:f + k] if k else x, 8 * k, 8 * n, f, sums[g])
    carry = torch.empty(sb, dtype=torch.uint8, device=x.device)
    tables, pays = [], []
    for g, (f, k) in enumerate(ranges):
        if g:
            lcf.lcf_dpratio_merge_summary_ptrs(sums[:g], g, carry)
        t, p, c = dp_compress_piece(x[f:f + k] if k else x[:0], n, f, carry if g else None, g)
        torch.cuda.synchronize()
        tables.append(t.cpu().numpy().tobytes())
        pays.append(p[:int(c.item())].cpu().numpy().tobytes())
    C = 2 * -(-n // TILE_WORDS)
    tab = b"".join(tables)
    assert len(tab) == 4 * C
    base = round16(HEADER + 4 * C)
    payload = b"".join(pays)
    hdr = (0x3146434C).to_bytes(4, "little") + bytes([1, 3, 8, 0]) + (8 * n).to_bytes(8, "little") + \
        C.to_bytes(8, "little") + len(payload).to_bytes(8, "little")
    return hdr + tab + bytes(base - HEADER - 4 * C) + payload


# ---- collectives and peer memory for the distributed DPratio calls ------------

def _is_gloo(group=None) -> bool:
    import torch.distributed as dist
    return dist.get_backend(group) == "gloo"


def _all_gather(t, group=None):
    """all_gather_into_tensor of a small tensor; with gloo the collective runs
    on a CPU copy (gloo has no CUDA all-gather-into-tensor)."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    src = t.cpu() if _is_gloo(group) else t
    out = torch.empty(world * src.numel(), dtype=src.dtype, device=src.device)
    dist.all_gather_into_tensor(out, src.contiguous().reshape(-1), group=group)
    return out.view((world,) + tuple(src.shape)).to(t.device)


def _barrier(group=None):
    import torch
    import torch.distributed as dist
    if torch.cuda.is_available():
        torch.cuda.synchronize()
    dist.barrier(group=group)


def gather_halo(x_shard, first_word: int, group=None):
    """The min(3, first_word) words before this rank's shard (FCM's hash
    context, L172): every rank contributes its last ≤ 3 words, and
    rank r takes the last words of ranks < r in order (a shard shorter than 3
    words, or empty, passes the earlier ranks' words through). One all-gather
    of 4 int64 per rank."""
    import torch
    import torch.distributed as dist
    rank = dist.get_rank(group)
    k = x_shard.numel()
    mine = torch.zeros(4, dtype=torch.int64, device=x_shard.device)
    c = min(3, k)
    mine[0] = c
    if c:
        mine[1:1 + c] = x_shard[k - c:].view(torch.int64)
    tails = _all_gather(mine, group).cpu()
    words = []
    for r in range(rank):
        cr = int(tails[r, 0])
        words.extend(int(v) for v in tails[r, 1:1 + cr])
    h = min(3, first_word)
    assert len(words) >= h, "shards must be given in array order"
    return torch.tensor(words[len(words) - h:], dtype=torch.int64, device=x_shard.device)


class PeerTensors:
    """Device pointers of every rank's copy of some tensors: this rank's own
    pointers, and its peers' mapped by CUDA IPC (lcf_ipc_export / import; over
    NVLink between GPUs, plain mappings on one GPU). The handles travel by
    all_gather_object. close() unmaps."""

    def __init__(self, tensors, group=None):
        import torch.distributed as dist
        from . import lcf
        self.rank, world = dist.get_rank(group), dist.get_world_size(group)
        mine = [lcf.lcf_ipc_export(t) for t in tensors]
        allh = [None] * world
        dist.all_gather_object(allh, mine, group=group)
        self.ptrs, self._opened = [], []
        for r in range(world):
            if r == self.rank:
                self.ptrs.append([t.data_ptr() for t in tensors])
            else:
                row = [lcf.lcf_ipc_import(h, off) for h, off in allh[r]]
                self._opened.extend(row)
                self.ptrs.append(row)

    def close(self):
        from . import lcf
        for p in self._opened:
            lcf.lcf_ipc_close(p)
        self._opened = []


def dp_compress_sharded(x_shard, n_total_words: int, first_word: int, group=None):
    """The distributed version (one process per GPU): the 3-word halo from the
    lower ranks, this rank's summary, its carry merged from the lower ranks'
    summaries read in place over CUDA IPC (no summary all-gather), its piece,
    and the payload-count exchange. Returns (table slice, payload piece,
    payload offset, total payload) with host ints."""
    import torch
    import torch.distributed as dist
    from . import lcf
    rank = dist.get_rank(group)
    halo = gather_halo(x_shard, first_word, group)
    h = halo.numel()
    # [halo ‖ shard] in one buffer, the shard's first word 16-byte aligned
    # (the allocation is: 4 words of headroom hold the ≤ 3 halo words)
    buf = torch.empty(4 + max(1, x_shard.numel()), dtype=torch.int64, device=x_shard.device)
    xs = buf[4:4 + x_shard.numel()]
    xs.copy_(x_shard.view(torch.int64))
    if h:
        buf[4 - h:4] = halo
    sb = lcf.lcf_dpratio_summary_bytes()
    mine = torch.empty(sb, dtype=torch.uint8, device=x_shard.device)
    nb = xs.numel() * 8
    lcf.lcf_dpratio_shard_summary(xs, nb, 8 * n_total_words, first_word, mine)
    _barrier(group)  # every summary written
    peers = PeerTensors([mine], group)
    carry = None
    if rank:
        carry = torch.empty(sb, dtype=torch.uint8, device=x_shard.device)
        lcf.lcf_dpratio_merge_summary_ptrs([peers.ptrs[r][0] for r in range(rank)], rank, carry)
    table, payload, count = dp_compress_piece(xs, n_total_words, first_word, carry, rank)
    _barrier(group)  # every merge has read the summaries
    peers.close()
    counts = _all_gather(count, group).reshape(-1).cpu().tolist()
    return table, payload[:counts[rank]], sum(counts[:rank]), sum(counts)


def dp_shard_substream(stream: bytes, world: int, rank: int) -> bytes:
    """Rank `rank`'s own LCF1 sub-stream of a DPratio stream: a header for its
    words, its size-table slice and its payload piece (what it holds after a
    sharded compression)."""
    import numpy as np
    h = np.frombuffer(stream[:32], np.uint64)
    n = int(h[1]) // 8
    C = int(h[2])
    table = np.frombuffer(stream[HEADER:HEADER + 4 * C], np.uint32)
    padded = (((table & 0x7FFFFFFF).astype(np.uint64) + 15) // 16) * 16
    offs = np.concatenate([[0], np.cumsum(padded)]).astype(np.uint64)
    base = round16(HEADER + 4 * C)
    f, k = dp_shard_words(n, world, rank)
    c0, c1 = 2 * (f // TILE_WORDS), 2 * (-(-(f + k) // TILE_WORDS))
    pay = stream[base + int(offs[c0]):base + int(offs[c1])]
    hdr = (0x3146434C).to_bytes(4, "little") + bytes([1, 3, 8, 0]) + (8 * k).to_bytes(8, "little") + \
        (c1 - c0).to_bytes(8, "little") + len(pay).to_bytes(8, "little")
    sub_base = round16(HEADER + 4 * (c1 - c0))
    return hdr + table[c0:c1].tobytes() + bytes(sub_base - HEADER - 4 * (c1 - c0)) + pay


def dp_simulate_decode_shards(stream: bytes, world: int):
    """Sharded DPratio decompression on one device: every shard decodes its
    sub-stream independently (words whose chains leave a tile that is not yet
    complete stay pending), then every shard finds its pending words' roots
    through the views of all shards, then every shard gathers the roots'
    values — the distributed protocol with the barriers as program order.
    Returns the int64 words."""
    import numpy as np
    import torch
    from . import lcf
    n = int(np.frombuffer(stream[8:16], np.uint64)[0]) // 8
    out = torch.empty(max(n, 1), dtype=torch.int64, device="cuda")
    views, subs = [], []
    for g in range(world):
        f, k = dp_shard_words(n, world, g)
        sub = torch.from_numpy(np.frombuffer(dp_shard_substream(stream, world, g), np.uint8).copy()).cuda()
        p = torch.empty(max(1, 2 * ((k + 31) // 32)), dtype=torch.int32, device="cuda")
        if k:
            lcf.lcf_dpratio_decompress_shard(sub, sub.numel(), f, out[f:f + k], 8 * k, p)
        subs.append(sub)
        views.append((f, k, out[f:f + k] if k else out, p))
    lcf.lcf_check_stream()
    for g in range(world):
        lcf.lcf_dpratio_find_roots(views, g)
    for g in range(world):
        lcf.lcf_dpratio_gather_roots(views, g)
    lcf.lcf_check_stream()
    return out[:n]


def dp_decompress_sharded(sub_stream, first_word: int, n_total: int, group=None):
    """The distributed sharded DPratio decompression of this rank's sub-stream
    (dp_shard_substream layout, CUDA uint8 tensor): decode with pending words,
    then the root resolution over every rank's words and bitmap, read in place
    over CUDA IPC (peer loads over NVLink; no message per pending word).
    Returns the rank's int64 words."""
    import torch
    import torch.distributed as dist
    from . import lcf
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    f, k = dp_shard_words(n_total, world, rank)
    assert f == first_word
    out = torch.empty(max(k, 1), dtype=torch.int64, device=sub_stream.device)
    pend = torch.zeros(max(1, 2 * ((k + 31) // 32)), dtype=torch.int32, device=sub_stream.device)
    if k:
        lcf.lcf_dpratio_decompress_shard(sub_stream, sub_stream.numel(), f, out, 8 * k, pend)
    lcf.lcf_check_stream()
    _barrier(group)  # a. every shard decoded
    peers = PeerTensors([out, pend], group)
    views = []
    for r in range(world):
        fr, kr = dp_shard_words(n_total, world, r)
        views.append((fr, kr, peers.ptrs[r][0], peers.ptrs[r][1]))
    lcf.lcf_dpratio_find_roots(views, rank)
    _barrier(group)  # c. every walk ended
    lcf.lcf_dpratio_gather_roots(views, rank)
    lcf.lcf_check_stream()
    _barrier(group)  # every peer read done before the mappings go
    peers.close()
    return out[:k]
