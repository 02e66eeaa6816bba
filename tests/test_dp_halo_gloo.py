"""Sharded DPratio (NEXT-1): the 3-word hash halo each rank needs before its
shard (sharded.gather_halo) with gloo, world 3 and 4, CPU tensors,
including empty and 1-word shards whose earlier ranks' words must pass
through. The halo must be exactly the array's words before the shard."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_azamifb25_b200 import sharded


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, lens, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        words = np.arange(1, sum(lens) + 1, dtype=np.int64) * 1000003
        f = sum(lens[:rank])
        shard = torch.from_numpy(words[f:f + lens[rank]].copy())
        halo = sharded.gather_halo(shard, f)
        q.put((rank, halo.tolist() == words[max(0, f - 3):f].tolist()))
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("lens", [[5, 0, 1, 4], [1, 1, 1], [0, 2, 7], [4096, 2048, 0, 2048]])
def test_gather_halo_gloo(lens):
    world = len(lens)
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, lens, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=30)
    assert all(ok is True for _, ok in res), res
