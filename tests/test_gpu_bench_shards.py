"""bench.py's weak-scaling inputs at N > 1 (make_fields): rank r's chunk-range
shard of the concatenated replicas, compressed on its own, must be exactly
that rank's piece of the 1-GPU stream of the concatenation, and
DPratio gets replica r whole. Run for N = 2 and 3 on one GPU, on the CESM
fields (25.9 MB, not a multiple of 16 KiB: shards cut through replicas)."""
import os
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("world", [2, 3])
def test_bench_weak_scaling_shards(world):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    sys.path.insert(0, ROOT)
    import bench
    from paper_conf_asplos_azamifb25_b200 import datagen, lcf, sharded
    sets = (("cesm_1800x3600_f32", ("U",), ("SPspeed", "SPratio")),)
    dev = torch.device("cuda", 0)
    per_rank = [bench.make_fields(world, r, dev, sets=sets) for r in range(world)]
    reps = [datagen.field("cesm_1800x3600_f32", "U", device=dev, replica=r).reshape(-1).view(torch.int32)
            for r in range(world)]
    whole = torch.cat(reps)
    total = whole.numel() * 4
    for ci, codec in enumerate(("SPspeed", "SPratio")):
        full = lcf.compress(codec, whole).cpu().numpy().tobytes()
        pieces = []
        for r in range(world):
            cfg, nm, c, x, tot = per_rank[r][ci]
            assert c == codec and tot == total
            first, k = sharded.shard_chunks(total, world, r)
            local = lcf.compress(codec, x)
            pb = int(np.frombuffer(local[24:32].cpu().numpy().tobytes(), np.uint64)[0])
            pieces.append(sharded.Piece(r, first, k, local, pb, 0, 0))
        assert sharded.assemble(codec, total, pieces) == full
