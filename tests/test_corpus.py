"""Corpus mode (BASELINE configs[4]): the corpus
composition, the whole-field assignment to ranks, and — with gloo on CPU,
world size 2, the CPU codec as the local codec — the single F-vector
exchange, checked field by field against the oracle."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_azamifb25_b200 import corpus

TINY = {"nyx_512x512x512_f32": (4, 32, 64), "hacc_280953867_f32": (9000,), "cesm_1800x3600_f32": (24, 200),
        "miranda_256x384x384_f64": (2, 24, 96)}


def test_corpus_composition():
    f = corpus.corpus_fields(1.0)
    by = {}
    for x in f:
        by.setdefault(x.config, []).append(x)
    assert [len(by[c]) for c, *_ in corpus.CATEGORIES] == [24, 12, 300, 114]
    f32 = sum(x.nbytes for x in f if x.codecs == corpus.SP_CODECS)
    f64 = sum(x.nbytes for x in f if x.codecs == corpus.DP_CODECS)
    assert 31 * 2**30 < f32 < 33.5 * 2**30 and 31 * 2**30 < f64 < 33 * 2**30  # ≈ 32 + 32 GiB
    assert len({(x.config, x.name, x.replica) for x in f}) == len(f)  # independent fields
    assert all(x.replica >= 1 for x in f)  # never the bench's own fields (replica 0)
    small = corpus.corpus_fields(1 / 64)
    assert {x.config for x in small} == set(by)


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_assignment_is_a_balanced_partition(world):
    f = corpus.corpus_fields(1.0)
    a = corpus.assign(f, world)
    assert sorted(i for r in a for i in r) == list(range(len(f)))
    assert a == corpus.assign(f, world)  # deterministic
    load = [sum(f[i].nbytes * len(f[i].codecs) for i in r) for r in a]
    biggest = max(x.nbytes * len(x.codecs) for x in f)
    assert max(load) - min(load) <= biggest


def _cpu_codec():
    from paper_conf_asplos_azamifb25_b200 import build, lcf_cpu
    build.build_cpu()

    def comp(codec, x):
        w = x.numpy().view(np.uint32 if x.dtype == torch.int32 else np.uint64)
        return torch.from_numpy(lcf_cpu.lcf_cpu_compress(codec, w, n_threads=2).copy())

    def dec(codec, s, like=None):
        y = lcf_cpu.lcf_cpu_decompress(codec, s.numpy(), n_threads=2)
        return torch.from_numpy(y.view(np.int32 if y.dtype == np.uint32 else np.int64).copy())
    return comp, dec


def _worker(rank, world, port, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        fields = corpus.corpus_fields(1 / 48, shapes=TINY)
        comp, dec = _cpu_codec()
        seen = []

        def check(f, codec, x, s):
            w = x.numpy().view(np.uint32 if x.dtype == torch.int32 else np.uint64)
            assert s.numpy().tobytes() == oracle.compress(codec, w), (f.fid, codec)
            seen.append((f.fid, codec, s.numel()))

        rep = corpus.run(fields, comp, dec, "cpu", rank, world, on_stream=check)
        mine = corpus.assign(fields, world)[rank]
        assert sorted({fid for fid, _, _ in seen}) == mine
        for fid, codec, n in seen:  # the all-reduced F-vector holds this rank's sizes
            assert rep["sizes"][2 * fid + fields[fid].codecs.index(codec)] == n
        assert all(v > 0 for v in rep["sizes"])  # every (field, codec) was done by some rank
        torch.save(rep, os.path.join(out_dir, f"rep{rank}.pt"))
    finally:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_corpus_gloo_two_ranks():
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(2, _free_port(), d), nprocs=2, join=True)
        r0, r1 = (torch.load(os.path.join(d, f"rep{r}.pt")) for r in (0, 1))
        assert r0["sizes"] == r1["sizes"] and r0["per_codec"] == r1["per_codec"]
        assert set(r0["per_codec"]) == {"SPspeed", "SPratio", "DPspeed", "DPratio"}
        assert r0["world"] == 2 and r0["gbs"] > 0


@pytest.mark.gpu
def test_corpus_gpu_tiny():
    """One rank on cuda:0, lcf as the codec: every stream equals the CPU codec's."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    comp, _ = _cpu_codec()

    def check(f, codec, x, s):
        assert s.cpu().numpy().tobytes() == comp(codec, x.cpu()).numpy().tobytes(), (f.fid, codec)

    fields = corpus.corpus_fields(1 / 48, shapes=TINY)
    gcomp, gdec, glen = corpus.lcf_codec()
    rep = corpus.run(fields, gcomp, gdec, "cuda", on_stream=check, length=glen)
    assert all(v > 0 for v in rep["sizes"]) and rep["gbs"] > 0
