"""Per-rank cost of sharded DPratio (NEXT-1) on one B200, for a Miranda-shaped
field cut into `world` tile ranges — what the last rank (a full carry, the
most pending words) runs, with the exchanges as they run on a node: the carry
merge reads the lower ranks' summaries through pointers (CUDA IPC on a node;
plain pointers here), and the decode's root pass walks every rank's words and
bitmaps through lcf_dp_view pointers. Only the barriers between the phases
and the NVLink latency of peer loads are missing.
Usage: python scripts/dp_shard_cost.py FIELD WORLD..."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf, sharded  # noqa: E402

field = sys.argv[1] if len(sys.argv) > 1 else "density"
worlds = [int(w) for w in sys.argv[2:]] or [2, 4, 8]
x = datagen.field("miranda_256x384x384_f64", field, device="cuda").reshape(-1).view(torch.int64)
n = x.numel()
sb = lcf.lcf_dpratio_summary_bytes()


def timed(fn, reps=5):
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts) * 1e3


full = lcf.compress("DPratio", x)
stream = full.cpu().numpy().tobytes()
cap = lcf.lcf_max_compressed_size("DPratio", None, 8 * n)
sbuf = torch.empty(cap, dtype=torch.uint8, device="cuda")
t_full_c = timed(lambda: lcf.lcf_compress("DPratio", None, x, 8 * n, sbuf, cap, sync=False))
y_full = torch.empty_like(x)
t_full_d = timed(lambda: lcf.lcf_decompress("DPratio", None, full, full.numel(), y_full, 8 * n, sync=False))
print(f"{field}: 1-GPU whole field compress {t_full_c:.0f} us, decompress {t_full_d:.0f} us")
for world in worlds:
    sums = [torch.empty(sb, dtype=torch.uint8, device="cuda") for _ in range(world)]
    carry = torch.empty(sb, dtype=torch.uint8, device="cuda")
    g = world - 1  # the last rank: a full carry
    f, k = sharded.dp_shard_words(n, world, g)
    for r in range(world):
        fr, kr = sharded.dp_shard_words(n, world, r)
        lcf.lcf_dpratio_shard_summary(x[fr:fr + kr], 8 * kr, 8 * n, fr, sums[r])
    t_sum = timed(lambda: lcf.lcf_dpratio_shard_summary(x[f:f + k], 8 * k, 8 * n, f, sums[g]))
    t_merge = timed(lambda: lcf.lcf_dpratio_merge_summary_ptrs(sums[:g], g, carry))
    t_comp = timed(lambda: sharded.dp_compress_piece(x[f:f + k], n, f, carry, g))

    def rank_seq():  # summary, merge over the peers' summaries, compress (the sort reused)
        lcf.lcf_dpratio_shard_summary(x[f:f + k], 8 * k, 8 * n, f, sums[g])
        lcf.lcf_dpratio_merge_summary_ptrs(sums[:g], g, carry)
        sharded.dp_compress_piece(x[f:f + k], n, f, carry, g)
    t_rank = timed(rank_seq)
    # decode: every shard decodes (the others' state is needed by the root pass), then the last rank's passes
    out = torch.empty(n, dtype=torch.int64, device="cuda")
    views, subs = [], []
    for r in range(world):
        fr, kr = sharded.dp_shard_words(n, world, r)
        sub = torch.from_numpy(np.frombuffer(sharded.dp_shard_substream(stream, world, r), np.uint8).copy()).cuda()
        p = torch.zeros(max(1, 2 * ((kr + 31) // 32)), dtype=torch.int32, device="cuda")
        subs.append(sub)
        views.append((fr, kr, out[fr:fr + kr], p))

    def decode_all():
        for r, (fr, kr, o, p) in enumerate(views):
            lcf.lcf_dpratio_decompress_shard(subs[r], subs[r].numel(), fr, o, 8 * kr, p)
    decode_all()
    t_dec = timed(lambda: lcf.lcf_dpratio_decompress_shard(subs[g], subs[g].numel(), f, views[g][2], 8 * k,
                                                           views[g][3]))

    def resolve():
        decode_all()
        for r in range(world):
            lcf.lcf_dpratio_find_roots(views, r)
        for r in range(world):
            lcf.lcf_dpratio_gather_roots(views, r)
    resolve()
    torch.cuda.synchronize()
    assert torch.equal(out, x)
    decode_all()
    for r in range(g):
        lcf.lcf_dpratio_find_roots(views, r)
    t_find = timed(lambda: lcf.lcf_dpratio_find_roots(views, g), reps=1)
    for r in range(g):
        lcf.lcf_dpratio_gather_roots(views, r)
    t_gather = timed(lambda: lcf.lcf_dpratio_gather_roots(views, g), reps=1)
    torch.cuda.synchronize()
    print(f"  world {world}: shard {8 * k / 1e6:.1f} MB | compress: summary {t_sum:.0f} us, merge (peer summaries) "
          f"{t_merge:.0f} us, compress {t_comp:.0f} us, the rank's sequence (sort reused) {t_rank:.0f} us | "
          f"decompress: shard decode {t_dec:.0f} us, find roots (peer views) {t_find:.0f} us, gather {t_gather:.0f} us")
