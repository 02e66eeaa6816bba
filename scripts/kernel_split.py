"""Per-kernel live timing (lcf_profile_enable / lcf_profile_report) of one
codec on one config field: median-free totals over --reps compress+decompress."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--codec", default="DPratio")
ap.add_argument("--config", default="miranda_256x384x384_f64")
ap.add_argument("--field", default="density")
ap.add_argument("--reps", type=int, default=10)
a = ap.parse_args()
x = datagen.field(a.config, a.field, device="cuda").reshape(-1)
x = x.view(torch.int32 if x.dtype == torch.float32 else torch.int64)
nb = x.numel() * x.element_size()
cap = lcf.lcf_max_compressed_size(a.codec, None, nb)
s = torch.empty(cap, dtype=torch.uint8, device="cuda")
y = torch.empty_like(x)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
n = lcf.lcf_compress(a.codec, None, x, nb, s, cap)
lcf.lcf_decompress(a.codec, None, s, n, y, nb)
torch.cuda.synchronize()
lcf.lcf_profile_report()
lcf.lcf_profile_enable(True)
for _ in range(a.reps):
    flush.fill_(1)
    lcf.lcf_compress(a.codec, None, x, nb, s, cap, sync=False)
    flush.fill_(1)
    lcf.lcf_decompress(a.codec, None, s, n, y, nb, sync=False)
torch.cuda.synchronize()
lcf.lcf_profile_enable(False)
rep = lcf.lcf_profile_report()
assert torch.equal(x, y) or os.environ.get("LCF_NOCHECK")
for k, (cnt, ms) in sorted(rep.items(), key=lambda kv: -kv[1][1]):
    print(f"{k:24s} launches/rep {cnt / a.reps:4.1f}  us/rep {1e3 * ms / a.reps:8.1f}")
