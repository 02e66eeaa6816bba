"""The multi-threaded CPU codec (liblcf_cpu.so) against
the oracle: byte-identical streams, exact round trips, the same accept/reject
decisions on corrupted streams, for every thread count. The GPU cross-check
(CPU stream == B200 stream, each decodes the other's) is marked gpu."""
import itertools

import numpy as np
import pytest

from paper_conf_asplos_azamifb25_b200 import datagen

ALGOS = ["SPspeed", "SPratio", "DPspeed", "DPratio"]


@pytest.fixture(scope="module")
def C():
    from paper_conf_asplos_azamifb25_b200 import build, lcf_cpu
    build.build_cpu()
    lcf_cpu.lib()
    return lcf_cpu


def wdt(algo):
    return np.uint32 if algo.startswith("SP") else np.uint64


def fdt(algo):
    return np.float32 if algo.startswith("SP") else np.float64


@pytest.mark.parametrize("algo", ALGOS)
def test_adversarial_parity(C, orc, algo):
    for name, words in datagen.adversarial(32 if algo.startswith("SP") else 64):
        ref = orc.compress(algo, words)
        for nt in (1, 3):
            s = C.lcf_cpu_compress(algo, words, n_threads=nt).tobytes()
            assert s == ref, f"{algo}/{name}/{nt} threads: stream differs from the oracle"
        assert np.array_equal(C.lcf_cpu_decompress(algo, ref, n_threads=2), words), name


@pytest.mark.parametrize("algo", ALGOS)
def test_smooth_and_tail_sizes(C, orc, algo):
    W = 32 if algo.startswith("SP") else 64
    CW = 16384 * 8 // W
    for n in (1, 31, 33, 127, 129, CW - 1, CW, CW + 1, 3 * CW + 1035):
        words = datagen.smooth_1d(n, fdt(algo), seed=n).view(wdt(algo))
        ref = orc.compress(algo, words)
        assert C.lcf_cpu_compress(algo, words, n_threads=4).tobytes() == ref, n
        assert np.array_equal(C.lcf_cpu_decompress(algo, ref, n_threads=4), words), n


def test_dpratio_matches_across_tiles(C, orc):
    """FCM distances inside a tile, across tiles and in chains (L197)."""
    y = datagen.smooth_1d(5 * 2048 + 77, np.float64, seed=5).view(np.uint64).copy()
    y[3000:3400] = y[100:500]      # matches into an earlier tile
    y[7000:7100] = y[6900:7000]    # in-tile repeats
    y[9000:9600] = y[8000:8600]    # chains (y[8000:8600] repeats the earlier run)
    y[8000:8600] = y[3000:3600]
    y[200:260] = 0                 # zero runs
    ref = orc.compress("DPratio", y)
    for nt in (1, 2, 7):
        assert C.lcf_cpu_compress("DPratio", y, n_threads=nt).tobytes() == ref
        assert np.array_equal(C.lcf_cpu_decompress("DPratio", ref, n_threads=nt), y)


@pytest.mark.parametrize("algo", ALGOS)
def test_exhaustive_tiny_streams(C, orc, algo):
    """Every 1- and 2-word stream over the 16-value special alphabet, plus
    every 3-word stream over its first 8 values."""
    sp = datagen.F32_SPECIALS if algo.startswith("SP") else datagen.F64_SPECIALS
    combos = list(itertools.product(range(16), repeat=1)) + list(itertools.product(range(16), repeat=2)) + \
        list(itertools.product(range(8), repeat=3))
    for combo in combos:
        words = sp[list(combo)]
        s = C.lcf_cpu_compress(algo, words, n_threads=1).tobytes()
        assert s == orc.compress(algo, words), combo
        assert np.array_equal(C.lcf_cpu_decompress(algo, s, n_threads=1), words), combo


def test_config_fields(C, orc):
    """A CESM-shaped f32 field (all 1583 chunks, ragged tail) and a Miranda slab."""
    x = datagen.field("cesm_1800x3600_f32", "U", device="cpu").numpy().reshape(-1).view(np.uint32)
    for algo in ("SPspeed", "SPratio"):
        ref = orc.compress(algo, x)
        s = C.lcf_cpu_compress(algo, x, n_threads=8)
        assert s.tobytes() == ref, algo
        assert np.array_equal(C.lcf_cpu_decompress(algo, s, n_threads=8), x)
    y = datagen.field("miranda_256x384x384_f64", "velocity", device="cpu", shape=(4, 384, 384))
    y = y.numpy().reshape(-1).view(np.uint64)
    for algo in ("DPspeed", "DPratio"):
        ref = orc.compress(algo, y)
        s = C.lcf_cpu_compress(algo, y, n_threads=8)
        assert s.tobytes() == ref, algo
        assert np.array_equal(C.lcf_cpu_decompress(algo, s, n_threads=8), y)


def test_empty_and_errors(C, orc):
    from paper_conf_asplos_azamifb25_b200.lcf import LcfError
    for algo in ALGOS:
        s = C.lcf_cpu_compress(algo, np.zeros(0, wdt(algo)))
        assert s.tobytes() == orc.compress(algo, np.zeros(0, wdt(algo)))
        assert C.lcf_cpu_decompress(algo, s).size == 0
    x = datagen.smooth_1d(3 * 4096, np.float32, seed=1).view(np.uint32)
    with pytest.raises(LcfError) as e:
        C.lcf_cpu_compress("SPspeed", x.view(np.uint8)[:-1])
    assert e.value.status == 1
    with pytest.raises(LcfError) as e:
        C.lcf_cpu_compress("SPspeed", x, dtype=1)
    assert e.value.status == 2
    s = C.lcf_cpu_compress("SPspeed", x)
    with pytest.raises(LcfError) as e:
        C.lcf_cpu_decompress("SPratio", s)
    assert e.value.status == 2
    with pytest.raises(LcfError) as e:
        C.lcf_cpu_decompress("SPspeed", s, out_capacity=100)
    assert e.value.status == 3


@pytest.mark.parametrize("algo", ALGOS)
def test_corruption_agrees_with_oracle(C, orc, algo):
    """Header, size-table and payload corruption: the CPU codec accepts exactly
    what the oracle accepts (FORMAT.md §7), and never crashes."""
    from paper_conf_asplos_azamifb25_b200.lcf import LcfError
    words = datagen.smooth_1d(3 * (16384 * 8 // (32 if algo.startswith("SP") else 64)) + 77, fdt(algo),
                              seed=3).view(wdt(algo))
    if algo == "DPratio":
        words = words.copy()
        words[5000:5100] = words[10:110]
    s = np.frombuffer(orc.compress(algo, words), np.uint8)
    rng = np.random.default_rng(7)
    for trial in range(150):
        t = s.copy()
        if trial < 20:
            pos = int(rng.integers(0, 32 + 4 * 8))
        else:
            pos = int(rng.integers(32, len(t)))
        t[pos] = int(rng.integers(0, 256))
        ok_orc = orc.decompress_status(algo, t.tobytes()) == 0
        try:
            y = C.lcf_cpu_decompress(algo, t, n_threads=3)
            ok = True
        except LcfError as e:
            assert e.status in (2, 3, 4)
            ok = False
        assert ok == ok_orc, (trial, pos)
        if ok:
            assert np.array_equal(y, orc.decompress(algo, t.tobytes()))
    with pytest.raises(LcfError):
        C.lcf_cpu_decompress(algo, s[:-16].copy())


@pytest.mark.gpu
@pytest.mark.parametrize("algo", ALGOS)
def test_cpu_codec_matches_gpu_stream(C, algo):
    """CPU/GPU compatibility (L41, L354): the B200 stream and the CPU codec's
    are the same bytes, and each side decodes the other's."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_azamifb25_b200 import lcf
    if algo.startswith("SP"):
        x = datagen.field("cesm_1800x3600_f32", "T", device="cuda").reshape(-1).view(torch.int32)
    else:
        x = datagen.field("miranda_256x384x384_f64", "density", device="cuda", shape=(16, 384, 384))
        x = x.reshape(-1).view(torch.int64)
    s_gpu = lcf.compress(algo, x)
    torch.cuda.synchronize()
    words = x.cpu().numpy().view(wdt(algo))
    s_cpu = C.lcf_cpu_compress(algo, words)
    assert s_gpu.cpu().numpy().tobytes() == s_cpu.tobytes()
    assert np.array_equal(C.lcf_cpu_decompress(algo, s_gpu.cpu().numpy()), words)
    y = lcf.decompress(algo, torch.from_numpy(s_cpu.copy()).cuda())
    assert torch.equal(y.reshape(-1), x)
