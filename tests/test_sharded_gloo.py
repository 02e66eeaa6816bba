"""Multi-process (gloo, CPU) tests of the sharded mode's host logic: chunk-range
partition, the single all-gather of payload byte counts, stream assembly.
The shard codec here is the oracle; on GPUs it is lcf_compress (same
contract, exercised by tests/test_gpu_sharded.py)."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_azamifb25_b200 import datagen, sharded


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _oracle_local(algo, shard):
    import oracle
    return torch.from_numpy(np.frombuffer(oracle.compress(algo, shard.numpy()), np.uint8).copy())


def _worker(rank, world, port, algo, n_words, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        dt = np.float32 if algo.startswith("SP") else np.float64
        words = datagen.smooth_1d(n_words, dt, seed=5)
        words[n_words // 3: n_words // 3 + 500] = np.random.default_rng(1).standard_normal(500)  # raw-ish chunk
        total = words.nbytes
        off, ln = sharded.shard_bytes(total, world, rank)
        shard = torch.from_numpy(words.view(np.uint8)[off:off + ln].copy().view(words.dtype))
        piece = sharded.compress_sharded(algo, shard, total, _oracle_local)
        # decode needs no exchange: the local stream decodes to the shard
        import oracle
        back = oracle.decompress(algo, piece.local_stream.numpy().tobytes())
        assert back.tobytes() == shard.numpy().tobytes()
        pieces = sharded.gather_pieces(piece)
        if rank == 0:
            stream = sharded.assemble(algo, total, pieces)
            ref = oracle.compress(algo, words)
            with open(os.path.join(out_dir, "result"), "w") as f:
                f.write("ok" if stream == ref else f"mismatch {len(stream)} {len(ref)}")
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("algo,world,n_words", [("SPspeed", 2, 9 * 4096 + 1035), ("SPratio", 2, 5 * 4096 + 33),
                                                ("DPspeed", 2, 7 * 2048 + 1), ("SPspeed", 3, 2 * 4096 + 7)])
def test_sharded_stream_identity_gloo(algo, world, n_words):
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(world, _free_port(), algo, n_words, d), nprocs=world, join=True)
        with open(os.path.join(d, "result")) as f:
            assert f.read() == "ok"


def test_shard_partition_covers_every_chunk_once():
    for n_bytes in [0, 4, 16384, 16384 * 7 + 12, 25920000, 1123815468]:
        for world in (1, 2, 3, 4, 8):
            C = sharded.num_chunks(n_bytes)
            seen, total = [], 0
            for r in range(world):
                first, k = sharded.shard_chunks(n_bytes, world, r)
                seen.extend(range(first, first + k))
                off, ln = sharded.shard_bytes(n_bytes, world, r)
                assert off == first * 16384 and (ln % 16384 == 0 or off + ln == n_bytes)
                total += ln
            assert seen == list(range(C)) and total == n_bytes


def test_dpratio_is_not_chunk_sharded():
    with pytest.raises(ValueError):
        sharded.compress_sharded("DPratio", None, 16, None)
