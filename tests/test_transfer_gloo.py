"""Compressed point-to-point transfer (NEXT-3, transfer.py): protocol and
stream equivalence on CPU — gloo, world size 2, the CPU codec as slice coder
(on B200s the same code runs lcf + NCCL; tests/test_gpu_parity.py checks the
GPU slice coder)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import fmt_ref
from paper_conf_asplos_azamifb25_b200 import datagen, transfer

CASES = [("SPspeed", np.float32), ("SPratio", np.float32), ("DPspeed", np.float64), ("DPratio", np.float64)]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _data(dt, seed):
    n = 9 * 16384 // np.dtype(dt).itemsize + 77  # 10 chunks, ragged tail
    w = datagen.smooth_1d(n, dt, seed=seed)
    w[1000:3000] = w[5]  # a constant stretch (FCM matches for DPratio)
    return w.view(np.uint32 if dt == np.float32 else np.uint64).copy()


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        res = []
        for i, (algo, dt) in enumerate(CASES):
            words = _data(dt, seed=30 + i)
            tw = torch.from_numpy(words.view(np.int32 if dt == np.float32 else np.int64))
            if rank == 0:
                st = transfer.send_compressed(tw, 1, algo, slice_bytes=3 * 16384)
                res.append((algo, st.wire_bytes, st.slices, st.n_bytes))
            else:
                got, st = transfer.recv_compressed(0, algo)
                res.append((algo, bool(torch.equal(got, tw)), st.wire_bytes, st.slices))
        q.put((rank, res))
    finally:
        dist.destroy_process_group()


def test_transfer_roundtrip_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    for (algo, wire_s, k_s, n_bytes), (algo_r, ok, wire_r, k_r) in zip(out[0], out[1]):
        assert algo == algo_r and ok, algo
        assert wire_s == wire_r and k_s == k_r
        assert k_s == (1 if algo == "DPratio" else 4)  # 3-chunk slices of a 10-chunk array
        assert wire_s < n_bytes  # smooth data with a constant stretch compresses


@pytest.mark.parametrize("algo,dt", CASES)
def test_substreams_equal_whole_stream(orc, algo, dt):
    """Concatenating the slices' table entries and payloads gives exactly the
    whole array's stream (chunk encodings are context-free, L104)."""
    words = _data(dt, seed=7)
    tw = torch.from_numpy(words.view(np.int32 if dt == np.float32 else np.int64))
    subs = transfer.substreams(tw, algo, codec=transfer.CpuCodec(), slice_bytes=3 * 16384)
    whole = orc.compress(algo, words)
    _, table, chunks = fmt_ref.parse_stream(whole)
    t2, c2 = [], []
    for s in subs:
        _, t, c = fmt_ref.parse_stream(s.numpy().tobytes())
        t2 += list(t)
        c2 += list(c)
    assert t2 == list(table) and c2 == list(chunks)
    for s in subs:
        assert transfer.substream_bytes(s[:32].numpy()) == s.numel()
