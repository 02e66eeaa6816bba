"""PCIe probe: pinned H2D / D2H copy bandwidth alone and concurrent (two
streams), and the host API's compress / decompress throughput on one field,
alone and with a concurrent partner call (the e2e pipeline's pairing)."""
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf  # noqa: E402

nb = 1 << 30
h1 = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
h2 = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
d1 = torch.empty(nb, dtype=torch.uint8, device="cuda")
d2 = torch.empty(nb, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def bw(fn, reps=3):
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        fn()
        torch.cuda.synchronize()
        ts.append(time.perf_counter() - t0)
    return min(ts)


t = bw(lambda: d1.copy_(h1, non_blocking=True))
print(f"H2D alone {nb / t / 1e9:.1f} GB/s")
t = bw(lambda: h1.copy_(d1, non_blocking=True))
print(f"D2H alone {nb / t / 1e9:.1f} GB/s")


def both():
    with torch.cuda.stream(s1):
        d1.copy_(h1, non_blocking=True)
    with torch.cuda.stream(s2):
        h2.copy_(d2, non_blocking=True)


t = bw(both)
print(f"H2D + D2H concurrent: {2 * nb / t / 1e9:.1f} GB/s total ({nb / t / 1e9:.1f} per direction)")

x = datagen.field("hacc_280953867_f32", "xx", device="cuda").reshape(-1).view(torch.int32)
n = x.numel() * 4
hx = torch.empty(n, dtype=torch.uint8, pin_memory=True)
hx.copy_(x.view(torch.uint8).cpu())
for codec in ("SPspeed", "SPratio"):
    cap = lcf.lcf_max_compressed_size(codec, None, n)
    hs = torch.empty(cap, dtype=torch.uint8, pin_memory=True)
    hs2 = torch.empty(cap, dtype=torch.uint8, pin_memory=True)
    hy = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    m = lcf.lcf_compress_host(codec, None, hx, n, hs, cap, stream=s1)
    t = bw(lambda: lcf.lcf_compress_host(codec, None, hx, n, hs2, cap, stream=s1))
    print(f"{codec} compress_host alone {n / t / 1e9:.1f} GB/s (ratio {n / m:.2f})")
    t = bw(lambda: lcf.lcf_decompress_host(codec, None, hs, m, hy, n, stream=s2))
    print(f"{codec} decompress_host alone {n / t / 1e9:.1f} GB/s")

    def pair():
        th = threading.Thread(target=lambda: lcf.lcf_compress_host(codec, None, hx, n, hs2, cap, stream=s1))
        th.start()
        lcf.lcf_decompress_host(codec, None, hs, m, hy, n, stream=s2)
        th.join()

    t = bw(pair)
    print(f"{codec} compress || decompress: {2 * n / t / 1e9:.1f} GB/s of fields")
