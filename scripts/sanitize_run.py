"""Small end-to-end run of all four codecs (and a corrupt stream) for
compute-sanitizer (memcheck / racecheck / synccheck / initcheck)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_asplos_azamifb25_b200 import datagen, lcf  # noqa: E402

for algo in ("SPspeed", "SPratio", "DPspeed", "DPratio"):
    W = 32 if algo.startswith("SP") else 64
    for name, words in datagen.adversarial(W)[:6] + [("smooth", datagen.smooth_1d(3 * 16384 // (W // 8) + 77,
                                                                               np.float32 if W == 32 else np.float64,
                                                                               seed=2).view(np.uint32 if W == 32 else np.uint64))]:
        x = torch.from_numpy(words.view(np.int32 if W == 32 else np.int64).copy()).cuda()
        s = lcf.compress(algo, x)
        y = lcf.decompress(algo, s)
        assert torch.equal(x, y), (algo, name)
        t = s.clone()
        t[min(40, t.numel() - 1)] ^= 0x5A  # corrupt a size entry / payload byte
        try:
            lcf.lcf_decompress(algo, None, t, t.numel(), y, y.numel() * y.element_size())
        except lcf.LcfError:
            pass
    print(algo, "ok")
torch.cuda.synchronize()
# multi-tile DPratio (several FCM sort tiles, rounds and decode tiles)
x = datagen.field("miranda_256x384x384_f64", "density", device="cuda", shape=(2, 384, 384)).reshape(-1).view(torch.int64)
s = lcf.compress("DPratio", x)
assert torch.equal(lcf.decompress("DPratio", s), x)
print("DPratio slab ok")
torch.cuda.synchronize()
# the sliced host-buffer path (3-chunk slices; DPratio: tile-range decodes)
os.environ["LCF_HOST_SLICE_BYTES"] = str(3 * 16384)
for algo in ("SPspeed", "SPratio", "DPspeed", "DPratio"):
    W = 32 if algo.startswith("SP") else 64
    dt = np.float32 if W == 32 else np.float64
    words = datagen.smooth_1d(12 * 16384 // (W // 8) + 77, dt, seed=5).view(np.uint32 if W == 32 else np.uint64).copy()
    words[3000:5000] = words[7]
    cap = lcf.lcf_max_compressed_size(algo, None, words.nbytes)
    hout = np.zeros(cap, np.uint8)
    n = lcf.lcf_compress_host(algo, None, words, words.nbytes, hout, cap)
    back = np.zeros_like(words)
    lcf.lcf_decompress_host(algo, None, hout, n, back, back.nbytes)
    assert np.array_equal(back, words), algo
    hout[40] ^= 0x5A
    try:
        lcf.lcf_decompress_host(algo, None, hout, n, back, back.nbytes)
    except lcf.LcfError:
        pass
    print(algo, "host slices ok")
torch.cuda.synchronize()
# sharded DPratio (NEXT-1): shard summaries / carries / pieces, and shard decodes with pending words
from paper_conf_asplos_azamifb25_b200 import sharded  # noqa: E402
w = datagen.field("miranda_256x384x384_f64", "density", shape=(1, 128, 384)).numpy().reshape(-1).view(np.uint64).copy()
w[5000:9000] = w[17]
xd = torch.from_numpy(w.view(np.int64)).cuda()
full = lcf.compress("DPratio", xd).cpu().numpy().tobytes()
assert sharded.dp_simulate_shards(xd, 3) == full
assert torch.equal(sharded.dp_simulate_decode_shards(full, 3), xd)
print("DPratio shards ok")
torch.cuda.synchronize()
# round 2: FCM-active DPratio (deferred candidates + verify, pending words,
# chain-node list walk/gather, the slow one-word match), and the multi-view
# root resolution of simulated shards
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from test_gpu_parity import fcm_stress_input  # noqa: E402
rt = datagen.field("miranda_256x384x384_f64", "rt_density", shape=(2, 64, 384)).numpy().reshape(-1).view(np.uint64)
base = np.random.default_rng(3).integers(0, 2**63, size=700, dtype=np.uint64)
for name, w in (("rt_slab", rt.copy()), ("fcm_stress", fcm_stress_input(n_const=20000)[:200000].copy()),
                ("period700", np.resize(base, 9 * 2048 + 5))):
    xd = torch.from_numpy(w.view(np.int64)).cuda()
    s = lcf.compress("DPratio", xd)
    assert torch.equal(lcf.decompress("DPratio", s), xd), name
    full = s.cpu().numpy().tobytes()
    assert torch.equal(sharded.dp_simulate_decode_shards(full, 3), xd), name
    t = s.clone()
    t[60] ^= 0x3C
    try:
        lcf.lcf_decompress("DPratio", None, t, t.numel(), xd.clone(), xd.numel() * 8)
        lcf.lcf_check_stream()
    except lcf.LcfError:
        pass
    print(name, "DPratio chains ok")
torch.cuda.synchronize()
