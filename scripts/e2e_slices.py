"""e2e (host-buffer API) time of the bench workload's compress+decompress per
slice size (LCF_HOST_SLICE_BYTES; 0 = the library's default)."""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf  # noqa: E402

jobs = []
for cfg, fields, codecs in (("cesm_1800x3600_f32", ("T", "U"), ("SPspeed", "SPratio")),
                            ("miranda_256x384x384_f64", ("density",), ("DPspeed", "DPratio"))):
    for f in fields:
        x = datagen.field(cfg, f).reshape(-1)
        for c in codecs:
            nb = x.numel() * x.element_size()
            hx = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
            hx.copy_(x.view(torch.uint8))
            cap = lcf.lcf_max_compressed_size(c, None, nb)
            jobs.append((c, nb, hx, torch.empty(cap, dtype=torch.uint8, pin_memory=True),
                         torch.empty(nb, dtype=torch.uint8, pin_memory=True), cap))
for sl in [int(a) for a in sys.argv[1:]] or [0]:
    if sl:
        os.environ["LCF_HOST_SLICE_BYTES"] = str(sl)
    else:
        os.environ.pop("LCF_HOST_SLICE_BYTES", None)
    ts = []
    for it in range(6):
        t0 = time.perf_counter()
        tot = 0
        for c, nb, hx, hs, hy, cap in jobs:
            n = lcf.lcf_compress_host(c, None, hx, nb, hs, cap)
            lcf.lcf_decompress_host(c, None, hs, n, hy, nb)
            tot += 2 * nb
        ts.append(time.perf_counter() - t0)
    t = statistics.median(ts[1:])
    print(f"slice {sl >> 20 if sl else 'default'} MiB: {t * 1e3:.1f} ms, {tot / t / 1e9:.1f} GB/s")
