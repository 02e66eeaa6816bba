"""NEXT-3, fused form: the sender's lcf_compress writes the stream straight
into the receiver's buffer through a CUDA IPC mapping (transfer.P2PChannel).
Two processes on cuda:0 (gloo for the handle and the signal; CUDA IPC maps the
receiver's buffer into the sender exactly as between two GPUs of a node). The
receiver's stream must equal the oracle's stream byte for byte, and its
decompressed words the sender's array — for all four codecs, twice over one
channel."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_asplos_azamifb25_b200 import datagen  # noqa: E402

CASES = {"SPspeed": 33 * 4096 + 17, "SPratio": 21 * 4096 + 5, "DPspeed": 30 * 2048 + 3, "DPratio": 25 * 2048 + 9}


def _words(algo, n, rep):
    dt = np.float32 if algo.startswith("SP") else np.float64
    w = datagen.smooth_1d(n, dt, seed=40 + rep).view(np.uint32 if dt == np.float32 else np.uint64).copy()
    if algo == "DPratio":
        w[n // 2:] = np.resize(w[:700], n - n // 2)  # FCM chains across tiles
    return w


def _worker(rank, port, q):
    import torch.distributed as dist
    import oracle
    from paper_conf_asplos_azamifb25_b200 import transfer
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=2)
    res = []
    try:
        for algo, n in CASES.items():
            ch = transfer.P2PChannel(0, 1, algo, 8 * n)
            for rep in range(2):
                w = _words(algo, n, rep)
                x = torch.from_numpy(w.view(np.int32 if w.dtype == np.uint32 else np.int64)).cuda()
                if rank == 0:
                    ch.send(x)
                else:
                    y = torch.empty_like(x)
                    nb = ch.recv(y, release=False)
                    torch.cuda.synchronize()
                    same_stream = ch.stream()[:nb].cpu().numpy().tobytes() == oracle.compress(algo, w)
                    ch.release()
                    res.append((algo, rep, same_stream, bool(torch.equal(x, y))))
            ch.close()
            dist.barrier()
        q.put((rank, res, None))
    except Exception as e:  # noqa: BLE001
        q.put((rank, res, repr(e)))
    finally:
        dist.destroy_process_group()


def test_p2p_channel_fused_compress_transfer():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=240) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
    for rank, res, err in out:
        assert err is None, f"rank {rank}: {err}"
    recv = out[1][1]
    assert len(recv) == 2 * len(CASES)
    for algo, rep, same_stream, same_words in recv:
        assert same_stream, f"{algo}/{rep}: stream differs from the oracle's"
        assert same_words, f"{algo}/{rep}: words differ"
