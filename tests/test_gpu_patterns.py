"""Every 2^32 f32 bit pattern in ONE 16 GiB stream, for SPspeed
and SPratio: the words are a fixed permutation of [0, 2^32)
(datagen.all_f32_patterns), compressed on the B200 in one lcf_compress call.
The whole stream is compared with the oracle's — chunk ranges on all host
cores, context-free chunks (L104) — piece by piece, and both sides are hashed
with SHA-256 (header ‖ size table ‖ pad ‖ payload); the stream decodes back to
the words. -m gpu; about a minute per codec."""
import hashlib
import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_asplos_azamifb25_b200 import datagen  # noqa: E402

N = 1 << 32
CW = 4096          # words per chunk
PIECE = 1 << 14    # chunks compared per piece (256 MiB of input)


@pytest.mark.parametrize("algo", ["SPspeed", "SPratio"])
def test_all_f32_patterns_one_stream(orc, algo):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_azamifb25_b200 import lcf
    x = torch.empty(N, dtype=torch.int32, device="cuda")
    step = 1 << 28
    for s in range(0, N, step):
        x[s:s + step] = datagen.all_f32_patterns(s, step, device="cuda")
    nb = 4 * N
    cap = lcf.lcf_max_compressed_size(algo, None, nb)
    st = torch.empty(cap, dtype=torch.uint8, device="cuda")
    n = lcf.lcf_compress(algo, None, x, nb, st, cap)
    C = N // CW
    table = st[32:32 + 4 * C].view(torch.int32).cpu().numpy().view(np.uint32)
    padded = ((table & 0x7FFFFFFF).astype(np.uint64) + 15) // 16 * 16
    offs = np.concatenate([[0], np.cumsum(padded)])
    base = (32 + 4 * C + 15) // 16 * 16
    assert n == base + int(offs[-1])
    hdr = np.frombuffer(st[:32].cpu().numpy().tobytes(), np.uint64)
    assert int(hdr[1]) == nb and int(hdr[2]) == C and int(hdr[3]) == int(offs[-1])
    assert not st[32 + 4 * C:base].cpu().numpy().any()
    # SHA-256 of the size table and of the payload, each side from its own bytes
    sha = {k: hashlib.sha256() for k in ("gpu_table", "gpu_payload", "orc_table", "orc_payload")}
    sha["gpu_table"].update(table.tobytes())
    nt = os.cpu_count() or 4

    def chunk_range(c0):
        w = datagen.all_f32_patterns(c0 * CW, PIECE * CW)
        return orc.compress_chunks(algo, w, 0, PIECE)

    with ThreadPoolExecutor(max_workers=nt) as ex:
        for p0 in range(0, C, PIECE * nt):
            starts = list(range(p0, min(C, p0 + PIECE * nt), PIECE))
            for c0, (tab, pay) in zip(starts, ex.map(chunk_range, starts)):
                assert np.array_equal(tab, table[c0:c0 + PIECE]), f"size table differs in chunks {c0}+"
                g = st[base + int(offs[c0]):base + int(offs[c0 + PIECE])].cpu().numpy().tobytes()
                assert g == pay, f"payload differs in chunks {c0}+"
                sha["orc_table"].update(tab.tobytes())
                sha["orc_payload"].update(pay)
                sha["gpu_payload"].update(g)
    d = {k: v.hexdigest() for k, v in sha.items()}
    assert d["gpu_table"] == d["orc_table"] and d["gpu_payload"] == d["orc_payload"]
    print(f"{algo}: 2^32 patterns, {n} B, table sha256 {d['gpu_table']}, payload sha256 {d['gpu_payload']}")
    y = torch.empty_like(x)
    lcf.lcf_decompress(algo, None, st, n, y, nb)
    assert torch.equal(x, y)
