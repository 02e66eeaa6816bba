"""Sharded mode on one GPU (-m gpu): shards compressed one after another with
lcf_compress / lcf_compress_shard must assemble into the 1-GPU stream, and the
NCCL count exchange runs through a single-rank process group."""
import os
import socket

import numpy as np
import pytest

from paper_conf_asplos_azamifb25_b200 import datagen, sharded

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def L():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_azamifb25_b200 import lcf
    lcf.lib()
    return lcf


def _words(algo, n, seed=3):
    dt = np.float32 if algo.startswith("SP") else np.float64
    w = datagen.smooth_1d(n, dt, seed=seed)
    return torch.from_numpy(w.view(np.int32 if dt == np.float32 else np.int64).copy()).cuda()


@pytest.mark.parametrize("algo", ["SPspeed", "SPratio", "DPspeed"])
@pytest.mark.parametrize("world", [2, 4, 8])
def test_local_streams_assemble_to_global(L, orc, algo, world):
    x = _words(algo, 37 * 4096 + 1035)
    total = x.numel() * x.element_size()
    full = L.compress(algo, x).cpu().numpy().tobytes()
    xb = x.view(torch.uint8)
    pieces, off_payload = [], 0
    for r in range(world):
        off, ln = sharded.shard_bytes(total, world, r)
        first, k = sharded.shard_chunks(total, world, r)
        shard = xb[off:off + ln].view(x.dtype)
        local = sharded.lcf_local_compress(algo, shard)
        pb = int(local[24:32].cpu().view(torch.int64).item())
        pieces.append(sharded.Piece(r, first, k, local, pb, off_payload, 0))
        off_payload += pb
        back = sharded.lcf_local_decompress(algo, local)  # no exchange on decode
        assert torch.equal(back, shard.view(back.dtype))
    assert sharded.assemble(algo, total, pieces) == full
    assert full == orc.compress(algo, x.cpu().numpy().view(np.uint32 if algo.startswith("SP") else np.uint64))


@pytest.mark.parametrize("algo", ["SPspeed", "SPratio", "DPspeed"])
def test_compress_shard_abi_matches_slices(L, algo):
    x = _words(algo, 21 * 4096 + 77, seed=4)
    total = x.numel() * x.element_size()
    full = L.compress(algo, x).cpu().numpy().tobytes()
    C = sharded.num_chunks(total)
    base = sharded.round16(32 + 4 * C)
    xb = x.view(torch.uint8)
    pos = base
    for world in (3,):
        pos = base
        for r in range(world):
            off, ln = sharded.shard_bytes(total, world, r)
            first, k = sharded.shard_chunks(total, world, r)
            table = torch.zeros(max(k, 1), dtype=torch.int32, device="cuda")
            cap = ln + 16 * max(k, 1) + 16
            pay = torch.zeros(cap, dtype=torch.uint8, device="cuda")
            cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
            L.lcf_compress_shard(algo, None, xb[off:off + ln], ln, total, first, table, pay, cap, cnt)
            n = int(cnt.item())
            assert table[:k].cpu().numpy().tobytes() == full[32 + 4 * first:32 + 4 * (first + k)]
            assert pay[:n].cpu().numpy().tobytes() == full[pos:pos + n]
            pos += n
        assert pos == len(full)
    hdr = torch.zeros(base, dtype=torch.uint8, device="cuda")
    L.lcf_write_header(algo, None, total, len(full) - base, hdr)
    assert hdr.cpu().numpy().tobytes()[:32] == full[:32]
    assert hdr.cpu().numpy().tobytes()[32 + 4 * C:base] == bytes(base - 32 - 4 * C)


def test_nccl_single_rank_exchange(L):
    import torch.distributed as dist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        x = _words("SPspeed", 9 * 4096 + 3)
        total = x.numel() * x.element_size()
        piece = sharded.compress_sharded("SPspeed", x, total, sharded.lcf_local_compress)
        stream = sharded.assemble("SPspeed", total, [piece])
        assert stream == L.compress("SPspeed", x).cpu().numpy().tobytes()
        # the distributed DPratio entry point (summary all-gather, count exchange) on one rank
        xd = _words("DPratio", 5 * 2048 + 17)
        table, payload, off, tot = sharded.dp_compress_sharded(xd, xd.numel(), 0)
        full = L.compress("DPratio", xd).cpu().numpy()
        C = 2 * 6
        base = (32 + 4 * C + 15) // 16 * 16
        assert off == 0 and tot == len(full) - base
        assert table.cpu().numpy().tobytes() == full[32:32 + 4 * C].tobytes()
        assert payload.cpu().numpy().tobytes() == full[base:].tobytes()
        # and the distributed decompression entry point on the same rank
        sub = torch.from_numpy(np.frombuffer(sharded.dp_shard_substream(full.tobytes(), 1, 0), np.uint8).copy()).cuda()
        assert torch.equal(sharded.dp_decompress_sharded(sub, 0, xd.numel()), xd)
    finally:
        dist.destroy_process_group()


def _dp_inputs():
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from test_gpu_parity import fcm_stress_input
    rng = np.random.default_rng(12)
    mixed = rng.integers(0, 2**63, size=40 * 2048 + 999, dtype=np.uint64)
    for _ in range(300):  # copies from anywhere earlier: matches that cross shard boundaries
        n = int(rng.integers(1, 40))
        i = int(rng.integers(n + 1, len(mixed) - n))
        j = int(rng.integers(0, i - n))
        mixed[i:i + n] = mixed[j:j + n]
    slab = datagen.field("miranda_256x384x384_f64", "density", shape=(2, 384, 384)).numpy().reshape(-1).view(np.uint64)
    rt = datagen.field("miranda_256x384x384_f64", "rt_density", shape=(4, 96, 384)).numpy().reshape(-1).view(np.uint64)
    return {"fcm_stress": fcm_stress_input(), "copies": mixed, "miranda_slab": slab.copy(), "rt_slab": rt.copy()}


@pytest.mark.parametrize("name", ["fcm_stress", "copies", "miranda_slab", "rt_slab"])
@pytest.mark.parametrize("world", [2, 3, 8])
def test_dpratio_shards_assemble_to_global(L, orc, name, world):
    """Sharded DPratio (NEXT-1): shard summaries → per-shard carries → shard
    pieces assemble into exactly the 1-GPU stream (and the oracle's)."""
    words = _dp_inputs()[name]
    x = torch.from_numpy(words.view(np.int64)).cuda()
    full = L.compress("DPratio", x).cpu().numpy().tobytes()
    got = sharded.dp_simulate_shards(x, world)
    assert got == full
    if name != "fcm_stress":
        assert got == orc.compress("DPratio", words)


@pytest.mark.parametrize("name", ["fcm_stress", "copies", "miranda_slab", "rt_slab"])
@pytest.mark.parametrize("world", [2, 3, 8])
def test_dpratio_shard_decode(L, name, world):
    """Sharded DPratio decompression (NEXT-1): each shard decodes its own
    sub-stream with chains leaving a tile left pending, then every shard
    finds its pending words' roots through all shards' views, then gathers
    them — the original words come back."""
    words = _dp_inputs()[name]
    x = torch.from_numpy(words.view(np.int64)).cuda()
    stream = L.compress("DPratio", x).cpu().numpy().tobytes()
    y = sharded.dp_simulate_decode_shards(stream, world)
    assert torch.equal(y, x)


def test_dpratio_shards_small_and_errors(L):
    """More ranks than tiles (empty shards), a ragged last tile, and argument
    checks of the sharded DPratio calls."""
    x = _words("DPratio", 2 * 2048 + 77)  # 3 tiles
    x[1000:1500] = x[3]
    full = L.compress("DPratio", x).cpu().numpy().tobytes()
    for world in (3, 5, 8):
        assert sharded.dp_simulate_shards(x, world) == full
        assert torch.equal(sharded.dp_simulate_decode_shards(full, world), x)
    sb = L.lcf_dpratio_summary_bytes()
    summ = torch.empty(sb, dtype=torch.uint8, device="cuda")
    n = x.numel()
    with pytest.raises(L.LcfError) as e:  # not tile-aligned
        L.lcf_dpratio_shard_summary(x[5:], 8 * (n - 5), 8 * n, 5, summ)
    assert e.value.status == 1
    with pytest.raises(L.LcfError) as e:  # a middle shard must be whole tiles
        L.lcf_dpratio_shard_summary(x, 8 * 100, 8 * n, 0, summ)
    assert e.value.status == 1
    with pytest.raises(L.LcfError) as e:  # payload capacity too small
        t = torch.empty(2, dtype=torch.int32, device="cuda")
        p = torch.empty(64, dtype=torch.uint8, device="cuda")
        c = torch.empty(1, dtype=torch.int64, device="cuda")
        L.lcf_dpratio_compress_shard(x[:2048], 8 * 2048, 8 * n, 0, None, t, p, 64, c)
    assert e.value.status == 3
