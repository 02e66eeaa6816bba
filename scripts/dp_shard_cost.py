"""Per-shard cost of sharded DPratio compression (NEXT-1) on one B200: the
summary call, the carry merge and the shard compress, for the Miranda density
field cut into `world` tile ranges (what each rank of a world-sized job runs,
minus the all-gathers)."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf, sharded  # noqa: E402

x = datagen.field("miranda_256x384x384_f64", "density", device="cuda").reshape(-1).view(torch.int64)
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


for world in [int(w) for w in sys.argv[1:]] or [8]:
    sums = torch.empty(world * sb, dtype=torch.uint8, device="cuda")
    carry = torch.empty(sb, dtype=torch.uint8, device="cuda")
    g = world - 1  # the last rank: a full carry
    f, k = sharded.dp_shard_words(n, world, g)
    for r in range(world):
        fr, kr = sharded.dp_shard_words(n, world, r)
        lcf.lcf_dpratio_shard_summary(x[fr:fr + kr], 8 * kr, 8 * n, fr, sums[r * sb:(r + 1) * sb])
    t_sum = timed(lambda: lcf.lcf_dpratio_shard_summary(x[f:f + k], 8 * k, 8 * n, f, sums[g * sb:(g + 1) * sb]))
    t_merge = timed(lambda: lcf.lcf_dpratio_merge_summaries(sums, g, carry))
    t_comp = timed(lambda: sharded.dp_compress_piece(x[f:f + k], n, f, carry, g))

    def rank_seq():  # what the rank runs: summary, merge, compress (the sort is reused)
        lcf.lcf_dpratio_shard_summary(x[f:f + k], 8 * k, 8 * n, f, sums[g * sb:(g + 1) * sb])
        lcf.lcf_dpratio_merge_summaries(sums, g, carry)
        sharded.dp_compress_piece(x[f:f + k], n, f, carry, g)
    t_rank = timed(rank_seq)
    t_full = timed(lambda: lcf.compress("DPratio", x)) if world == int(sys.argv[1] if len(sys.argv) > 1 else 8) else 0
    print(f"world {world}: shard {8 * k / 1e6:.1f} MB: summary {t_sum:.0f} us, merge {t_merge:.0f} us, "
          f"compress {t_comp:.0f} us; the rank's sequence (sort reused) {t_rank:.0f} us "
          f"(1-GPU whole field {t_full:.0f} us)")
