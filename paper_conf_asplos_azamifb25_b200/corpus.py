"""Corpus mode: BASELINE.json configs[4] ("all four codecs on a 64 GB mixed
float32/float64 synthetic corpus sharded across 2/4/8 B200"), SURVEY §8(d)
config 5 and §8(e).

The corpus (§8(d)):
  f32 ≈ 32 GiB: 24 NYX-like 512³ fields, 12 HACC-like 280,953,867-word arrays,
                300 CESM-like 1800×3600 fields — SPspeed and SPratio on each;
  f64 ≈ 32 GiB: 114 Miranda-like 256×384×384 fields (density, velocity and
                the FCM-active rt_density in turn) — DPspeed and DPratio.
Every field is its own LCF1 stream, generated on whichever rank owns it from
its field id (replica ≥ 1: independent of the bench's fields). `scale` keeps a
proportional prefix of each category (at least one field each).

Multi-GPU (one process per GPU): fields are assigned whole to ranks by a
deterministic longest-processing-time rule (per-field stream identity holds
trivially; DPratio's FCM is a whole-array pass, L104, so it is never split).
The only exchanges are one all-reduce of the F-vector of compressed sizes
(each entry written by its owner, §8(e): "corpus mode batches all fields'
counts into one allgather of an F-vector") and one max of the device times.
Aggregate GB/s = Σ uncompressed bytes of all (field, codec) compressions and
decompressions ÷ max over ranks of the device time.

The codec is a parameter (`lcf.compress`/`lcf.decompress` on GPUs); the CPU
tests pass the CPU codec (liblcf_cpu.so) to exercise the assignment and the
exchange with gloo. Run: `python -m paper_conf_asplos_azamifb25_b200.corpus
--scale 0.125` (torchrun for N > 1).
"""
from __future__ import annotations

import argparse
import json
import os
import time
from dataclasses import dataclass, field

from . import datagen

SP_CODECS = ("SPspeed", "SPratio")
DP_CODECS = ("DPspeed", "DPratio")

# (config, field names alternating, count at scale 1, codecs)
CATEGORIES = (
    ("nyx_512x512x512_f32", ("velocity", "baryon_density"), 24, SP_CODECS),
    ("hacc_280953867_f32", ("xx", "vx"), 12, SP_CODECS),
    ("cesm_1800x3600_f32", ("T", "U"), 300, SP_CODECS),
    ("miranda_256x384x384_f64", ("density", "velocity", "rt_density"), 114, DP_CODECS),
)


@dataclass
class FieldSpec:
    fid: int
    config: str
    name: str
    replica: int
    codecs: tuple
    shape: tuple | None = None  # a sub-block (tests); None = the config's full shape
    nbytes: int = field(default=0)

    def __post_init__(self):
        cid, full, dtype, _ = datagen.CONFIGS[self.config]
        n = 1
        for d in (self.shape or full):
            n *= d
        self.nbytes = n * (4 if dtype is datagen.torch.float32 else 8)


def corpus_fields(scale: float = 1.0, shapes: dict | None = None) -> list:
    """The corpus's field list (deterministic order; fid = position)."""
    out = []
    for config, names, count, codecs in CATEGORIES:
        k = max(1, int(round(count * scale)))
        for j in range(k):
            out.append(FieldSpec(len(out), config, names[j % len(names)], 1 + j, codecs,
                                 (shapes or {}).get(config)))
    return out


def assign(fields: list, world: int) -> list:
    """Longest processing time first onto the least-loaded rank (ties: lowest
    rank), weight = bytes × codecs; returns per-rank lists of fids."""
    load = [0] * world
    owned = [[] for _ in range(world)]
    for f in sorted(fields, key=lambda f: (-f.nbytes * len(f.codecs), f.fid)):
        r = min(range(world), key=lambda r: (load[r], r))
        owned[r].append(f.fid)
        load[r] += f.nbytes * len(f.codecs)
    return [sorted(o) for o in owned]


def _word_view(x):
    import torch
    return x.reshape(-1).view(torch.int32 if x.dtype == torch.float32 else torch.int64)


def lcf_codec():
    """The B200 codec for run(): stream-ordered calls with no host round trip
    inside the timed region (the stream buffer is passed whole; its length is
    read from its own header on the device)."""
    import torch

    from . import lcf

    def comp(codec, x):
        nb = x.numel() * x.element_size()
        cap = lcf.lcf_max_compressed_size(codec, None, nb)
        s = torch.empty(cap, dtype=torch.uint8, device=x.device)
        lcf.lcf_compress(codec, None, x, nb, s, cap, sync=False)
        return s

    def dec(codec, s, like):
        y = torch.empty_like(like)
        lcf.lcf_decompress(codec, None, s, s.numel(), y, y.numel() * y.element_size(), sync=False)
        return y

    def length(s):  # round16(32 + 4·n_chunks) + payload_bytes (FORMAT.md §1)
        c, p = s[16:24].view(torch.int64), s[24:32].view(torch.int64)
        return ((32 + 4 * c + 15) // 16) * 16 + p

    return comp, dec, length


def run(fields: list, compress, decompress, device, rank: int = 0, world: int = 1, group=None,
        verify: bool = True, on_stream=None, length=None) -> dict:
    """Compress and decompress this rank's fields with every codec of each.
    `compress(codec, x) -> stream`, `decompress(codec, stream, like) -> x`
    (tensors on `device`), `length(stream)` → its byte count (default numel).
    Device time: CUDA events around each call on a CUDA device, else wall
    clock. Returns the corpus report (identical on every rank)."""
    import torch
    import torch.distributed as dist
    mine = assign(fields, world)[rank]
    fvec = torch.zeros(2 * len(fields), dtype=torch.int64, device=device)  # compressed bytes per (field, codec)
    cuda = torch.device(device).type == "cuda"
    ms = 0.0
    by_codec = {}
    # warm-up outside the timing: each codec once on its largest field here
    # (library workspaces are sized by the largest call and then reused)
    for codec in sorted({c for i in mine for c in fields[i].codecs}):
        big = max((fields[i] for i in mine if codec in fields[i].codecs), key=lambda f: (f.nbytes, -f.fid))
        x = _word_view(datagen.field(big.config, big.name, device=device, replica=big.replica, shape=big.shape))
        decompress(codec, compress(codec, x), x)
        del x
    if cuda:
        torch.cuda.synchronize()
    for fid in mine:
        f = fields[fid]
        x = _word_view(datagen.field(f.config, f.name, device=device, replica=f.replica, shape=f.shape))
        for ci, codec in enumerate(f.codecs):
            if cuda:
                torch.cuda.synchronize()
                e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
                e[0].record()
                s = compress(codec, x)
                e[1].record()
                y = decompress(codec, s, x)
                e[2].record()
                torch.cuda.synchronize()
                tc, td = e[0].elapsed_time(e[1]), e[1].elapsed_time(e[2])
            else:
                t0 = time.perf_counter()
                s = compress(codec, x)
                t1 = time.perf_counter()
                y = decompress(codec, s, x)
                t2 = time.perf_counter()
                tc, td = 1e3 * (t1 - t0), 1e3 * (t2 - t1)
            if verify:
                assert torch.equal(y.reshape(-1), x), f"corpus field {fid} ({f.config}/{f.name}) {codec}: round trip"
            n = length(s) if length is not None else s.numel()
            n = int(n)
            if on_stream is not None:
                on_stream(f, codec, x, s[:n])
            fvec[2 * fid + ci] = n
            ms += tc + td
            d = by_codec.setdefault(codec, [0, 0, 0.0, 0.0])
            d[0] += f.nbytes
            d[1] += n
            d[2] += tc
            d[3] += td
        del x
    # the exchanges: the F-vector (each entry has one owner) and the max device time
    t = torch.tensor([ms], dtype=torch.float64, device=device)
    if world > 1:
        dist.all_reduce(fvec, group=group)
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
        allc = sorted({c for f in fields for c in f.codecs})  # per-codec sums over ranks
        vec = torch.zeros(4 * len(allc), dtype=torch.float64, device=device)
        for i, c in enumerate(allc):
            if c in by_codec:
                vec[4 * i:4 * i + 4] = torch.tensor(by_codec[c], dtype=torch.float64, device=device)
        dist.all_reduce(vec, group=group)
        by_codec = {c: vec[4 * i:4 * i + 4].tolist() for i, c in enumerate(allc)}
    sizes = fvec.cpu().tolist()
    total_in = sum(f.nbytes * len(f.codecs) for f in fields)
    total_ms = float(t.item())
    report = {
        "fields": len(fields), "bytes": sum(f.nbytes for f in fields), "world": world,
        "gbs": 2 * total_in / total_ms / 1e6 if total_ms > 0 else None, "max_rank_ms": total_ms,
        "per_codec": {c: {"ratio": v[0] / v[1] if v[1] else None, "compress_gbs": v[0] / v[2] / 1e6 if v[2] else None,
                          "decompress_gbs": v[0] / v[3] / 1e6 if v[3] else None, "bytes": int(v[0])}
                      for c, v in by_codec.items()},
        "sizes": sizes,
    }
    return report


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=float, default=0.125)
    ap.add_argument("--no-verify", action="store_true")
    args = ap.parse_args()
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    fields = corpus_fields(args.scale)
    comp, dec, length = lcf_codec()
    rep = run(fields, comp, dec, dev, rank, world, verify=not args.no_verify, length=length)
    if rank == 0:
        rep.pop("sizes")
        print(json.dumps({"metric": "corpus compress+decompress throughput (uncompressed GB/s)",
                          "scale": args.scale, **rep}))
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
