"""Sharded DPratio decompression (NEXT-1): the cross-rank resolution of
pending words (sharded.dp_resolve_pending_distributed) with gloo, world 3 and
4, CPU tensors. Each rank holds a decoded shard in which some words are pending
on a global index of an earlier shard — which may itself be pending, so chains
cross several shards. The result must equal resolving the whole array in
index order."""
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


def _case(n, world, seed):
    """(values, pending mask, targets) for the whole array, and the resolved
    words: a pending word i copies word target[i] < first word of its shard."""
    rng = np.random.default_rng(seed)
    vals = rng.integers(0, 2**62, size=n, dtype=np.int64)
    pend = np.zeros(n, bool)
    tgt = np.zeros(n, np.int64)
    for r in range(1, world):
        f, k = sharded.dp_shard_words(n, world, r)
        for i in rng.choice(k, size=min(k, 40), replace=False):
            pend[f + i] = True
            tgt[f + i] = rng.integers(0, f)  # any earlier shard (maybe a pending word itself)
    final = vals.copy()
    for i in range(n):  # index order: targets are final when read
        if pend[i]:
            final[i] = final[tgt[i]]
    return vals, pend, tgt, final


def _worker(rank, world, port, n, seed, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        vals, pend, tgt, final = _case(n, world, seed)
        f, k = sharded.dp_shard_words(n, world, rank)
        out = torch.from_numpy(np.where(pend[f:f + k], tgt[f:f + k], vals[f:f + k]).copy())
        bits = np.zeros((k + 31) // 32 * 32, bool)
        bits[:k] = pend[f:f + k]
        words = np.packbits(bits.reshape(-1, 8)[:, ::-1], axis=1).reshape(-1).view("<u4").astype(np.int64)
        pb = torch.from_numpy(words.astype(np.uint32).view(np.int32).copy())
        sharded.dp_resolve_pending_distributed(out, pb, f, n)
        q.put((rank, bool(np.array_equal(out.numpy(), final[f:f + k]))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [3, 4])
def test_resolve_pending_gloo(world):
    n = 11 * 2048 + 333
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, 5 + world, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    assert all(res.values()), res
