"""Run one codec on one config field a few times (for ncu captures)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--codec", default="SPspeed")
ap.add_argument("--config", default="nyx_512x512x512_f32")
ap.add_argument("--field", default="velocity")
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
x = datagen.field(a.config, a.field, device="cuda").reshape(-1)
x = x.view(torch.int32 if x.dtype == torch.float32 else torch.int64)
nb = x.numel() * x.element_size()
cap = lcf.lcf_max_compressed_size(a.codec, None, nb)
s = torch.empty(cap, dtype=torch.uint8, device="cuda")
y = torch.empty_like(x)
for _ in range(a.reps):
    n = lcf.lcf_compress(a.codec, None, x, nb, s, cap)
    lcf.lcf_decompress(a.codec, None, s, n, y, nb)
torch.cuda.synchronize()
assert torch.equal(x, y)
print(a.codec, a.config, a.field, nb, n, nb / n)
