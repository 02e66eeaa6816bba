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
    finally:
        dist.destroy_process_group()
