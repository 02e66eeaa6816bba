"""Per-chunk pipeline trace of a speed-codec compress (globaltimer stamps from
lcf__trace_compress): where does a chunk's latency go, and how busy is the
pipeline over time? The stamps exist only in a library built with
-DLCF_TRACE=1 (e.g. `scripts/build_variants.sh` with that define, then
LCF_LIB_PATH=build/variants/<name>.so)."""
import argparse
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--codec", default="SPspeed")
ap.add_argument("--config", default="cesm_1800x3600_f32")
ap.add_argument("--field", default="T")
a = ap.parse_args()
x = datagen.field(a.config, a.field, device="cuda").reshape(-1)
x = x.view(torch.int32 if x.dtype == torch.float32 else torch.int64)
nb = x.numel() * x.element_size()
C = lcf.lcf_num_chunks(a.codec, nb)
cap = lcf.lcf_max_compressed_size(a.codec, None, nb)
s = torch.empty(cap, dtype=torch.uint8, device="cuda")
tr = torch.zeros(C * 8, dtype=torch.int64, device="cuda")
L = lcf.lib()
f = L.lcf__trace_compress
f.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_size_t,
              ctypes.c_void_p, ctypes.c_void_p]
for _ in range(3):
    tr.zero_()
    st = f(lcf.ALGOS[a.codec], lcf.ALGO_DTYPE[lcf.ALGOS[a.codec]], x.data_ptr(), nb, s.data_ptr(), cap, tr.data_ptr(),
           torch.cuda.current_stream().cuda_stream)
    assert st == 0
torch.cuda.synchronize()
t = tr.view(C, 8).cpu().numpy().astype(np.float64)
t0 = t[:, 0].min()
t = (t - t0) / 1e3  # µs since the first ticket
names = ["ticket", "data", "published", "slot", "packed", "storer", "lookback", "stored"]
print(f"{a.codec} {a.config}/{a.field}: {C} chunks, span {t[:, 7].max():.1f} us (first ticket → last store read)")
groups = [("all", t)] if a.codec != "DPratio" else [("V chunks", t[0::2]), ("Dist chunks", t[1::2])]
for label, tg in groups:
    if len(groups) > 1:
        print(f" {label}:")
    for k in range(1, 8):
        d = tg[:, k] - tg[:, k - 1]
        print(f"  {names[k - 1]:>9s} → {names[k]:<9s}: median {np.median(d):7.2f} us  p90 {np.percentile(d, 90):7.2f}  max {d.max():7.2f}")
for q in (0, 0.1, 0.5, 0.9, 1.0):
    print(f"  ticket time quantile {q:.1f}: {np.quantile(t[:, 0], q):7.2f} us; stored: {np.quantile(t[:, 7], q):7.2f} us")
