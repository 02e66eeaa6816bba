"""A/B timing of library variants: median CUDA-event time of compress and
decompress of one config field (LCF_LIB_PATH selects the library)."""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--codec", default="DPspeed")
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
ct, dt = [], []
for _ in range(a.reps):
    for lst, fn in ((ct, lambda: lcf.lcf_compress(a.codec, None, x, nb, s, cap, sync=False)),
                    (dt, lambda: lcf.lcf_decompress(a.codec, None, s, n, y, nb, sync=False))):
        flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        lst.append(e0.elapsed_time(e1))
assert torch.equal(x, y)
c, d = statistics.median(ct), statistics.median(dt)
moved = nb + n
print(f"{os.path.basename(os.environ.get('LCF_LIB_PATH', 'liblcf.so')):18s} {a.codec} {a.config}/{a.field} "
      f"comp {c * 1e3:7.1f} us {nb / c / 1e6:7.1f} GB/s ({moved / c / 1e6 / 6459.3:5.1%})  "
      f"decomp {d * 1e3:7.1f} us {nb / d / 1e6:7.1f} GB/s ({moved / d / 1e6 / 6459.3:5.1%})  ratio {nb / n:.3f}")
