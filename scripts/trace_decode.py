"""Per-tile trace of a DPratio decompress (globaltimer stamps from the
diagnostic entry point lcf__trace_decompress): where a tile's time goes."""
import argparse
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="miranda_256x384x384_f64")
ap.add_argument("--field", default="density")
a = ap.parse_args()
x = datagen.field(a.config, a.field, device="cuda").reshape(-1).view(torch.int64)
nb = x.numel() * 8
cap = lcf.lcf_max_compressed_size("DPratio", None, nb)
s = torch.empty(cap, dtype=torch.uint8, device="cuda")
n = lcf.lcf_compress("DPratio", None, x, nb, s, cap)
T = (x.numel() + 2047) // 2048
y = torch.empty_like(x)
tr = torch.zeros(T * 8, dtype=torch.int64, device="cuda")
f = lcf.lib().lcf__trace_decompress
f.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_size_t,
              ctypes.c_void_p, ctypes.c_void_p]
for _ in range(3):
    tr.zero_()
    st = f(lcf.ALGOS["DPratio"], lcf.ALGO_DTYPE[lcf.ALGOS["DPratio"]], s.data_ptr(), n, y.data_ptr(), nb,
           tr.data_ptr(), torch.cuda.current_stream().cuda_stream)
    assert st == 0
torch.cuda.synchronize()
assert torch.equal(x, y)
t = tr.view(T, 8).cpu().numpy().astype(np.float64)
t = (t - t[:, 0].min()) / 1e3
names = ["ticket", "slot", "data", "released", "V done", "Dist done", "FCM done", "stored"]
print(f"DPratio decode {a.config}/{a.field}: {T} tiles, span {t[:, 7].max():.1f} us")
for k in range(1, 8):
    d = t[:, k] - t[:, k - 1]
    print(f"  {names[k - 1]:>9s} → {names[k]:<9s}: median {np.median(d):7.2f} us  p90 {np.percentile(d, 90):7.2f}")
