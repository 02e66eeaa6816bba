"""Distributed sharded DPratio (NEXT-1) with real processes: 2 and 3 ranks on
cuda:0 (gloo for the barriers and the handle exchange; every box here has one
GPU, and NCCL refuses two ranks on one device). Peer memory goes through the
library's CUDA IPC calls, as between GPUs of one node. Each rank holds only
its own shard: the 3-word halo comes from the lower ranks, the
carry from the lower ranks' summaries read in place, and the decode resolves
chains through every rank's words. The assembled stream must be the 1-GPU
stream byte for byte and the decoded words the input."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_asplos_azamifb25_b200 import datagen, sharded  # noqa: E402


def _input(name):
    if name == "rt":
        x = datagen.field("miranda_256x384x384_f64", "rt_density", shape=(3, 64, 384)).numpy().reshape(-1)
        return x.view(np.int64).copy()
    rng = np.random.default_rng(5)
    w = rng.integers(0, 2**63, size=9 * 2048 + 700, dtype=np.int64)
    for _ in range(200):  # copies from anywhere earlier, across shard boundaries
        n = int(rng.integers(3, 30))
        i = int(rng.integers(n + 1, len(w) - n))
        j = int(rng.integers(0, i - n))
        w[i:i + n] = w[j:j + n]
    return w


def _worker(rank, world, port, name, q):
    import torch.distributed as dist
    from paper_conf_asplos_azamifb25_b200 import lcf
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        words = _input(name)
        n = len(words)
        f, k = sharded.dp_shard_words(n, world, rank)
        x_shard = torch.from_numpy(words[f:f + k].copy()).cuda()  # this rank holds only its shard
        table, payload, off, tot = sharded.dp_compress_sharded(x_shard, n, f)
        torch.cuda.synchronize()
        pieces = [None] * world
        dist.all_gather_object(pieces, (table.cpu().numpy().tobytes(), payload.cpu().numpy().tobytes(), off))
        C = 2 * -(-n // 2048)
        tab = b"".join(p[0] for p in pieces)
        pay = b"".join(p[1] for p in pieces)
        base = (32 + 4 * C + 15) // 16 * 16
        hdr = (0x3146434C).to_bytes(4, "little") + bytes([1, 3, 8, 0]) + (8 * n).to_bytes(8, "little") + \
            C.to_bytes(8, "little") + len(pay).to_bytes(8, "little")
        stream = hdr + tab + bytes(base - 32 - 4 * C) + pay
        full = lcf.compress("DPratio", torch.from_numpy(words).cuda()).cpu().numpy().tobytes()
        same = stream == full and off == sum(len(p[1]) for p in pieces[:rank]) and tot == len(pay)
        sub = torch.from_numpy(np.frombuffer(sharded.dp_shard_substream(full, world, rank), np.uint8).copy()).cuda()
        y = sharded.dp_decompress_sharded(sub, f, n)
        ok = bool(np.array_equal(y.cpu().numpy(), words[f:f + k]))
        q.put((rank, same, ok, None))
    except Exception as e:  # noqa: BLE001
        q.put((rank, False, False, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name", ["rt", "copies"])
@pytest.mark.parametrize("world", [2, 3])
def test_distributed_dpratio_ipc(name, world):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=600) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    for rank, same, ok, err in res:
        assert err is None, f"rank {rank}: {err}"
        assert same, f"rank {rank}: assembled stream differs from the 1-GPU stream"
        assert ok, f"rank {rank}: decoded words differ"
