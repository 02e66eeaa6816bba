"""GPU parity: the sm_100a path (through the C ABI) vs the CPU oracle, bit-exact
on streams, size tables and decompressed bits (-m gpu)."""
import os

import numpy as np
import pytest

import fmt_ref
from paper_conf_asplos_azamifb25_b200 import datagen

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

SPEED_ALGOS = ["SPspeed", "DPspeed"]
GPU_ALGOS = ["SPspeed", "DPspeed", "SPratio", "DPratio"]


@pytest.fixture(scope="module")
def L():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_asplos_azamifb25_b200 import lcf
    lcf.lib()
    return lcf


def wdt(algo):
    return np.uint32 if algo.startswith("SP") else np.uint64


def tdt(algo):
    return torch.int32 if algo.startswith("SP") else torch.int64


def to_dev(words: np.ndarray):
    t = torch.from_numpy(words.view(np.int32 if words.dtype == np.uint32 else np.int64).copy())
    return t.cuda()


def gpu_roundtrip(L, algo, x_dev):
    s = L.compress(algo, x_dev)
    y = L.decompress(algo, s)
    torch.cuda.synchronize()
    return s.cpu().numpy().tobytes(), y


def check_parity(L, orc, algo, words: np.ndarray, name=""):
    words = np.ascontiguousarray(words).reshape(-1)
    x = to_dev(words)
    s_gpu, y = gpu_roundtrip(L, algo, x)
    s_orc = orc.compress(algo, words)
    if s_gpu != s_orc:
        h1, t1, c1 = fmt_ref.parse_stream(s_gpu)
        h2, t2, c2 = fmt_ref.parse_stream(s_orc)
        bad = [i for i in range(min(len(t1), len(t2))) if t1[i] != t2[i] or c1[i] != c2[i]]
        raise AssertionError(f"{algo}/{name}: stream differs (len {len(s_gpu)} vs {len(s_orc)}; "
                             f"headers {h1 == h2}; first bad chunk {bad[:5]})")
    assert torch.equal(y.reshape(-1), x.reshape(-1)), f"{algo}/{name}: decompressed bits differ"
    # cross-decode: oracle decodes the GPU stream (identical bytes) and GPU decodes oracle's
    assert np.array_equal(orc.decompress(algo, s_gpu), words)
    return len(s_gpu)


def test_all_codecs_built(L):
    """Every codec runs on the device: a missing one fails here instead of
    silently skipping its parity suite."""
    for a in GPU_ALGOS:
        x = torch.zeros(16, dtype=tdt(a), device="cuda")
        s = L.compress(a, x)
        assert torch.equal(L.decompress(a, s), x), a


@pytest.mark.parametrize("algo", GPU_ALGOS)
def test_adversarial_parity(L, orc, algo):
    for name, words in datagen.adversarial(32 if algo.startswith("SP") else 64):
        check_parity(L, orc, algo, words, name)


@pytest.mark.parametrize("algo", GPU_ALGOS)
def test_exhaustive_tiny_parity(L, orc, algo):
    """Every 1-, 2- and 3-word stream over the 16 special values:
    16 + 256 + 4096 streams per codec, GPU = oracle byte for byte."""
    import itertools
    sp = datagen.F32_SPECIALS if algo.startswith("SP") else datagen.F64_SPECIALS
    for r in (1, 2, 3):
        for combo in itertools.product(range(16), repeat=r):
            check_parity(L, orc, algo, sp[list(combo)], f"tiny{combo}")


@pytest.mark.parametrize("algo", GPU_ALGOS)
def test_random_width_subchunks(L, orc, algo):
    """Every MPLG width 0..W (both flag states) and ragged tails."""
    W = 32 if algo.startswith("SP") else 64
    dt = wdt(algo)
    rng = np.random.default_rng(W)
    SW = 4096 // W
    CW = 32 * SW
    for n in (CW * 3 + 1035, SW * 7 + 5, CW):
        u = np.zeros(n, dtype=dt)  # the DIFFMS output we want the encoder to see
        for s in range(-(-n // SW)):
            w = int(rng.integers(0, W + 1))
            m = min(SW, n - s * SW)
            vals = rng.integers(0, 2**W - 1, size=m, dtype=dt, endpoint=True)
            u[s * SW:s * SW + m] = vals & dt((1 << w) - 1) if w < W else vals
        d = (u >> dt(1)) ^ (dt(0) - (u & dt(1)))  # magnitude-sign → two's complement
        words = np.concatenate([np.cumsum(d[c:c + CW], dtype=dt) for c in range(0, n, CW)])
        check_parity(L, orc, algo, words, f"widths{n}")


CONFIG_CASES = [("SPspeed", "tiny_512x512_f32", "f"), ("SPratio", "tiny_512x512_f32", "f"),
                ("SPspeed", "cesm_1800x3600_f32", "T"), ("SPspeed", "cesm_1800x3600_f32", "U"),
                ("SPratio", "cesm_1800x3600_f32", "T"), ("SPratio", "cesm_1800x3600_f32", "U")]


@pytest.mark.parametrize("algo,config,field", CONFIG_CASES)
def test_config_field_parity(L, orc, algo, config, field):
    x = datagen.field(config, field, device="cuda")
    words = x.cpu().numpy().view(wdt(algo))
    n = check_parity(L, orc, algo, words, f"{config}/{field}")
    assert n < words.nbytes  # these smooth fields compress


@pytest.mark.parametrize("algo,field", [("DPspeed", "density"), ("DPspeed", "velocity"),
                                        ("DPratio", "density"), ("DPratio", "velocity")])
def test_miranda_subvolume_parity(L, orc, algo, field):
    """Miranda-shaped f64 (a 32×384×384 slab of the full field, 4.7 M words)."""
    x = datagen.field("miranda_256x384x384_f64", field, device="cuda", origin=(0, 0, 0), shape=(32, 384, 384))
    check_parity(L, orc, algo, x.cpu().numpy().view(np.uint64), f"miranda/{field}")


def test_dpratio_mixed_match_tiles(L, orc):
    """Tiles with and without FCM matches interleaved (the encoder's all-zero
    Dist fast path and its per-CTA cached stream alternate with the general
    path), plus a ragged last tile."""
    x = datagen.field("miranda_256x384x384_f64", "density", shape=(2, 384, 384)).numpy().reshape(-1).view(np.uint64)
    x = x[: 2048 * 100 + 777].copy()
    T = 2048
    for t in range(3, 100, 3):  # every third tile repeats an earlier stretch: matches
        src = (t - 3) * T + 100
        x[t * T: t * T + 1500] = x[src: src + 1500]
    x[50 * T + 10: 50 * T + 20] = x[50 * T + 9]  # a short constant run inside a matching-free tile
    check_parity(L, orc, "DPratio", x, "mixed_match_tiles")


def test_dpratio_raw_tiles_with_matches(L, orc):
    """Random-bit tiles (V and Dist chunks stored raw) that still carry FCM
    matches: copied 16-word runs from random earlier positions, copies of
    copies (chains across tiles), and a ragged last tile. Exercises the
    decoder's raw-V + FCM path and cross-tile chain resolution."""
    rng = np.random.default_rng(11)
    T = 2048
    x = rng.integers(0, 2**63, size=12 * T + 333, dtype=np.uint64)
    for t in range(2, 13):
        run = 16 if t % 2 else 6  # even tiles: two short runs only, so V stays incompressible (raw)
        for _ in range(40 if t % 2 else 2):
            i = t * T + int(rng.integers(0, T - run))
            if i + run > len(x):
                continue
            j = int(rng.integers(0, i - run))
            x[i:i + run] = x[j:j + run]
    _, table, _ = fmt_ref.parse_stream(orc.compress("DPratio", x))
    assert any(e >> 31 for e in table[::2]), "expected raw V chunks"
    check_parity(L, orc, "DPratio", x, "raw_tiles_with_matches")


def fcm_stress_input(n_const=300_000, seed=5):
    """FCM inputs with long same-hash runs and matches at every candidate depth:
      - a constant run: one hash for every position, every match at distance 1;
      - period-50 random values: 50 hashes, each recurring every 50 positions
        (matches at distance 50);
      - one context (a, b, c) followed by a value cycling with period 3, 4 or 5:
        the match is the 3rd or 4th same-hash candidate, or none (5 > 4, L174);
      - noise between the blocks."""
    rng = np.random.default_rng(seed)
    parts = [np.full(n_const, 0x400921FB54442D18, dtype=np.uint64)]
    per = rng.integers(0, 2**63, size=50, dtype=np.uint64)
    parts.append(np.tile(per, 12_000))
    ctx = rng.integers(0, 2**63, size=3, dtype=np.uint64)
    for cyc in (3, 4, 5):
        vals = rng.integers(0, 2**63, size=cyc, dtype=np.uint64)
        blk = np.empty((20_000, 4), dtype=np.uint64)
        blk[:, :3] = ctx
        blk[:, 3] = vals[np.arange(20_000) % cyc]
        parts.append(blk.reshape(-1))
        parts.append(rng.integers(0, 2**63, size=5_000, dtype=np.uint64))
    return np.concatenate(parts)


def test_dpratio_fcm_long_hash_runs(L, orc):
    """FCM distances over long same-hash runs (one hash for 300 K positions,
    50 hashes recurring every 50 positions, matches at the 3rd/4th candidate
    or beyond the window) — stream identical to the oracle's."""
    check_parity(L, orc, "DPratio", fcm_stress_input(), "fcm_long_hash_runs")


def oracle_pieces_threaded(orc, algo, words, n_chunks, per=256):
    """The oracle's size table and padded payload for chunks [0, n_chunks) of
    `words`, computed in chunk ranges on all host cores (the oracle's own
    compress_chunks; ctypes releases the GIL). Chunks are context-free (L104),
    so the concatenated pieces are the oracle's whole-stream table and payload."""
    from concurrent.futures import ThreadPoolExecutor
    ranges = [(c, min(per, n_chunks - c)) for c in range(0, n_chunks, per)]
    with ThreadPoolExecutor(max_workers=os.cpu_count() or 4) as ex:
        parts = list(ex.map(lambda r: orc.compress_chunks(algo, words, r[0], r[1]), ranges))
    return np.concatenate([t for t, _ in parts]), b"".join(p for _, p in parts)


def full_stream_parity(L, orc, algo, x_dev):
    """Full-size check: the whole GPU stream equals the oracle's byte for byte
    (header fields, every size-table entry, every payload byte), and decodes."""
    s = L.compress(algo, x_dev)
    stream = s.cpu().numpy()
    words = x_dev.cpu().numpy().reshape(-1).view(wdt(algo))
    C = L.lcf_num_chunks(algo, words.nbytes)
    table, payload = oracle_pieces_threaded(orc, algo, words, C)
    hdr = np.frombuffer(stream[:32].tobytes(), np.uint64)
    algo_id = {"SPspeed": 0, "SPratio": 1, "DPspeed": 2, "DPratio": 3}[algo]
    assert stream[:8].tobytes() == (0x3146434C).to_bytes(4, "little") + bytes([1, algo_id, words.itemsize, 0])
    assert int(hdr[1]) == words.nbytes and int(hdr[2]) == C and int(hdr[3]) == len(payload)
    assert np.array_equal(stream[32:32 + 4 * C].view(np.uint32), table)
    base = (32 + 4 * C + 15) // 16 * 16
    assert not stream[32 + 4 * C:base].any()
    assert len(stream) == base + len(payload)
    assert stream[base:].tobytes() == payload
    y = L.decompress(algo, s)
    assert torch.equal(y, x_dev.reshape(-1))
    return len(stream)


@pytest.mark.parametrize("algo,config,field", [
    ("SPspeed", "nyx_512x512x512_f32", "baryon_density"), ("SPspeed", "nyx_512x512x512_f32", "velocity"),
    ("SPspeed", "hacc_280953867_f32", "xx"), ("SPspeed", "hacc_280953867_f32", "vx"),
    ("SPratio", "nyx_512x512x512_f32", "baryon_density"), ("SPratio", "nyx_512x512x512_f32", "velocity"),
    ("SPratio", "hacc_280953867_f32", "xx"), ("SPratio", "hacc_280953867_f32", "vx"),
    ("DPspeed", "miranda_256x384x384_f64", "density"), ("DPspeed", "miranda_256x384x384_f64", "rt_density")])
def test_full_size_stream_parity(L, orc, algo, config, field):
    """BASELINE configs[2]/[3] at full size, the bench's fields: whole streams
    byte for byte against the oracle (sampled chunks were not
    enough)."""
    x = datagen.field(config, field, device="cuda").reshape(-1)
    x = x.view(tdt(algo))
    full_stream_parity(L, orc, algo, x)
    del x
    torch.cuda.empty_cache()


@pytest.mark.parametrize("field", ["density", "rt_density"])
def test_full_size_dpratio_stream(L, orc, field):
    """The bench's DPratio workload at full size (Miranda-shaped 256×384×384
    f64, 37.7 M words: 2304 FCM sort tiles, 18,432 encode tiles) — density
    (no FCM match) and rt_density (about half the words match, every match
    chaining back through all earlier rows): the whole GPU stream equals the
    oracle's byte for byte (the oracle needs ~1 min), and it decodes back,
    also through the host-buffer path."""
    x = datagen.field("miranda_256x384x384_f64", field, device="cuda").reshape(-1).view(torch.int64)
    s = L.compress("DPratio", x)
    hx = x.cpu().numpy().view(np.uint64)
    ref = orc.compress("DPratio", hx)
    assert s.numel() == len(ref)
    assert np.array_equal(s.cpu().numpy(), np.frombuffer(ref, np.uint8))
    assert torch.equal(L.decompress("DPratio", s), x)
    # the host-buffer path compresses in tile slices with carried FCM state and
    # decodes in tile ranges: the same bytes, the same words
    hout = np.zeros(L.lcf_max_compressed_size("DPratio", None, hx.nbytes), np.uint8)
    nh = L.lcf_compress_host("DPratio", None, hx, hx.nbytes, hout, hout.nbytes)
    assert nh == len(ref) and hout[:nh].tobytes() == ref
    hy = np.zeros_like(hx)
    assert L.lcf_decompress_host("DPratio", None, hout, nh, hy, hy.nbytes) == hx.nbytes
    assert np.array_equal(hy, hx)
    del x, s
    torch.cuda.empty_cache()


def test_dpratio_long_chains(L, orc, monkeypatch):
    """FCM decode on chains that cross many tiles (L197): a constant array
    (every word copies its predecessor: one chain through the whole array), a
    period-384 array (chains of row length), a period-5000 array (each hop
    crosses tiles) and an rt_density slab — GPU stream = oracle, words back,
    also through 3-tile host slices."""
    rng = np.random.default_rng(3)
    base = rng.integers(0, 2**63, size=5000, dtype=np.uint64)
    cases = {"constant": np.full(40 * 2048 + 5, 0x400921FB54442D18, np.uint64),
             "period384": np.resize(base[:384], 30 * 2048 + 100),
             "period5000": np.resize(base, 30 * 2048 + 7)}
    rt = datagen.field("miranda_256x384x384_f64", "rt_density", shape=(3, 64, 384)).numpy().reshape(-1)
    cases["rt_slab"] = rt.view(np.uint64).copy()
    monkeypatch.setenv("LCF_HOST_SLICE_BYTES", str(3 * 16384))
    for name, w in cases.items():
        check_parity(L, orc, "DPratio", w, name)
        ref = orc.compress("DPratio", w)
        back = np.zeros_like(w)
        assert L.lcf_decompress_host("DPratio", None, np.frombuffer(ref, np.uint8).copy(), len(ref), back,
                                     back.nbytes) == w.nbytes
        assert np.array_equal(back, w), name
@pytest.mark.parametrize("algo", SPEED_ALGOS)
def test_async_path_and_corruption(L, orc, algo):
    words = datagen.smooth_1d(3 * 4096 + 77, np.float32 if algo == "SPspeed" else np.float64, seed=3)
    words = words.view(wdt(algo))
    x = to_dev(words)
    s = L.compress(algo, x)
    out = torch.empty_like(x)
    # async: no out_bytes, then check
    L.lcf_decompress(algo, None, s, s.numel(), out, out.numel() * out.element_size(), sync=False)
    L.lcf_check_stream()
    assert torch.equal(out, x)
    # header corruption → CORRUPT_STREAM, both sync and async
    for off, val in [(0, 0), (6, 3), (16, 99), (24, 255)]:
        t = s.clone()
        t[off] = val
        with pytest.raises(L.LcfError) as e:
            L.lcf_decompress(algo, None, t, t.numel(), out, out.numel() * out.element_size())
        assert e.value.status == 4
        L.lcf_decompress(algo, None, t, t.numel(), out, out.numel() * out.element_size(), sync=False)
        with pytest.raises(L.LcfError):
            L.lcf_check_stream()
    # size-table corruption: reject, never crash; random payload bytes: no crash
    t = s.clone()
    t[32 + 3] = 0x7F
    with pytest.raises(L.LcfError):
        L.lcf_decompress(algo, None, t, t.numel(), out, out.numel() * out.element_size())
    rng = np.random.default_rng(1)
    for _ in range(50):
        t = s.clone()
        pos = int(rng.integers(32, s.numel()))
        t[pos] = int(rng.integers(0, 256))
        try:
            L.lcf_decompress(algo, None, t, t.numel(), out, out.numel() * out.element_size())
            ok_gpu = True
        except L.LcfError:
            ok_gpu = False
        ok_orc = orc.decompress_status(algo, t.cpu().numpy().tobytes()) == 0
        assert ok_gpu == ok_orc
    # too small an output buffer
    with pytest.raises(L.LcfError) as e:
        L.lcf_decompress(algo, None, s, s.numel(), out, 100)
    assert e.value.status == 3
    torch.cuda.synchronize()


@pytest.mark.parametrize("algo", SPEED_ALGOS)
def test_concurrent_streams_and_repeats(L, orc, algo):
    """Different streams get separate workspaces; repeated calls stay exact."""
    dt = np.float32 if algo == "SPspeed" else np.float64
    xs = [to_dev(datagen.smooth_1d(50 * 4096 // (1 if dt == np.float32 else 2) + i, dt, seed=i).view(wdt(algo)))
          for i in range(3)]
    expect = [orc.compress(algo, x.cpu().numpy().view(wdt(algo))) for x in xs]
    streams = [torch.cuda.Stream() for _ in xs]
    for rep in range(5):
        outs = []
        for x, st in zip(xs, streams):
            with torch.cuda.stream(st):
                cap = L.lcf_max_compressed_size(algo, None, x.numel() * x.element_size())
                o = torch.empty(cap, dtype=torch.uint8, device="cuda")
                L.lcf_compress(algo, None, x, x.numel() * x.element_size(), o, cap, sync=False, stream=st)
                outs.append(o)
        torch.cuda.synchronize()
        for o, e in zip(outs, expect):
            assert o[:len(e)].cpu().numpy().tobytes() == e


def test_empty_and_info(L, orc):
    for algo in ["SPspeed", "DPspeed"]:
        x = torch.zeros(0, dtype=tdt(algo), device="cuda")
        s = L.compress(algo, x)
        assert s.cpu().numpy().tobytes() == orc.compress(algo, np.zeros(0, wdt(algo)))
        info = L.lcf_get_info(s, s.numel())
        assert info["uncompressed_bytes"] == 0 and info["compressed_bytes"] == 32
        assert L.decompress(algo, s).numel() == 0


def test_host_buffer_api(L, orc):
    words = datagen.smooth_1d(10 * 4096 + 3, np.float32, seed=8).view(np.uint32)
    cap = L.lcf_max_compressed_size("SPspeed", None, words.nbytes)
    hout = np.zeros(cap, np.uint8)
    n = L.lcf_compress_host("SPspeed", None, words, words.nbytes, hout, cap)
    assert hout[:n].tobytes() == orc.compress("SPspeed", words)
    back = np.zeros_like(words)
    m = L.lcf_decompress_host("SPspeed", None, hout, n, back, back.nbytes)
    assert m == words.nbytes and np.array_equal(back, words)


def test_host_api_two_threads(L, orc, monkeypatch):
    """The host API from two threads at once, each on its own CUDA stream (the
    bench's e2e pipeline: one thread compresses while the other decompresses):
    per-stream workspaces keep the calls independent — every stream equals the
    oracle's and every field comes back bit-exact, over sliced host paths."""
    import threading
    monkeypatch.setenv("LCF_HOST_SLICE_BYTES", str(5 * 16384))
    fields = []
    for k, algo in enumerate(("SPspeed", "SPratio", "DPspeed", "DPratio") * 2):
        dt = np.float32 if algo.startswith("SP") else np.float64
        w = datagen.smooth_1d(24 * 16384 // np.dtype(dt).itemsize + 37 * k, dt, seed=40 + k).view(wdt(algo)).copy()
        if algo == "DPratio":
            w[3000:] = np.resize(w[:2500], w.size - 3000)  # FCM matches across host slices
        fields.append((algo, w, orc.compress(algo, w)))
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    errors = []

    def worker(t):
        try:
            for rep in range(3):
                for algo, w, ref in fields[t::2]:
                    cap = L.lcf_max_compressed_size(algo, None, w.nbytes)
                    hout = np.zeros(cap, np.uint8)
                    n = L.lcf_compress_host(algo, None, w, w.nbytes, hout, cap, stream=streams[t])
                    assert hout[:n].tobytes() == ref, (algo, rep)
                    back = np.zeros_like(w)
                    assert L.lcf_decompress_host(algo, None, hout, n, back, back.nbytes, stream=streams[t]) == w.nbytes
                    assert np.array_equal(back, w), (algo, rep)
        except BaseException as e:
            errors.append(e)

    ths = [threading.Thread(target=worker, args=(t,)) for t in range(2)]
    for th in ths:
        th.start()
    for th in ths:
        th.join()
    assert not errors, errors


@pytest.mark.parametrize("algo", GPU_ALGOS)
def test_host_pipelined_slices(L, orc, algo, monkeypatch):
    """The sliced host path (3-chunk slices: 14 slices and a ragged tail; for
    DPratio 3-tile decode slices whose FCM distances reach into earlier slices)
    writes the oracle's stream, decodes it and the oracle's, and accepts/rejects
    corrupted streams exactly as the oracle does."""
    monkeypatch.setenv("LCF_HOST_SLICE_BYTES", str(3 * 16384))
    dt = np.float32 if algo.startswith("SP") else np.float64
    words = datagen.smooth_1d(40 * 16384 // np.dtype(dt).itemsize + 77, dt, seed=21).view(wdt(algo)).copy()
    words[5000:9000] = words[100]  # a constant stretch (small MPLG widths / zero RZE bytes)
    cap = L.lcf_max_compressed_size(algo, None, words.nbytes)
    hout = np.zeros(cap, np.uint8)
    n = L.lcf_compress_host(algo, None, words, words.nbytes, hout, cap)
    ref = orc.compress(algo, words)
    assert hout[:n].tobytes() == ref
    back = np.zeros_like(words)
    assert L.lcf_decompress_host(algo, None, hout, n, back, back.nbytes) == words.nbytes
    assert np.array_equal(back, words)
    with pytest.raises(L.LcfError) as e:  # the stitched stream must fit
        L.lcf_compress_host(algo, None, words, words.nbytes, hout, n - 1)
    assert e.value.status == 3
    rng = np.random.default_rng(4)
    for trial in range(40):
        t = np.frombuffer(ref, np.uint8).copy()
        pos = int(rng.integers(32, len(ref))) if trial % 4 else int(rng.integers(32, 32 + 4 * 41))
        t[pos] ^= np.uint8(1 << int(rng.integers(0, 8)))
        try:
            L.lcf_decompress_host(algo, None, t, len(t), back, back.nbytes)
            ok_gpu = True
        except L.LcfError:
            ok_gpu = False
        assert ok_gpu == (orc.decompress_status(algo, t.tobytes()) == 0), (trial, pos)
        if ok_gpu:
            assert np.array_equal(back, orc.decompress(algo, t.tobytes()))


@pytest.mark.parametrize("algo", GPU_ALGOS)
def test_transfer_gpu_slices(L, orc, algo):
    """NEXT-3 slice coder on the B200: the sub-streams send_compressed puts on
    the wire equal the oracle's streams of the same slices (and the CPU
    codec's), and decoding them slice by slice (the receiver's path, loopback
    without a second GPU) restores the array."""
    from paper_conf_asplos_azamifb25_b200 import transfer
    dt = np.float32 if algo.startswith("SP") else np.float64
    words = datagen.smooth_1d(20 * 16384 // np.dtype(dt).itemsize + 77, dt, seed=33).view(wdt(algo)).copy()
    words[2000:6000] = words[9]
    x = to_dev(words)
    subs = transfer.substreams(x, algo, slice_bytes=3 * 16384)
    ref = transfer.substreams(torch.from_numpy(words.view(np.int32 if dt == np.float32 else np.int64)), algo,
                              codec=transfer.CpuCodec(), slice_bytes=3 * 16384)
    assert [s.cpu().numpy().tobytes() for s in subs] == [r.numpy().tobytes() for r in ref]
    wb = words.itemsize
    bounds = list(transfer._slices(words.nbytes, wb, 3 * 16384 if algo != "DPratio" else transfer._whole(words.nbytes)))
    assert [s.cpu().numpy().tobytes() for s in subs] == [orc.compress(algo, words[w0:w1]) for w0, w1 in bounds]
    out = torch.empty_like(x)
    codec = transfer.GpuCodec()
    assert len(bounds) == len(subs)
    for (w0, w1), s in zip(bounds, subs):
        codec.decompress_into(transfer._algo_id(algo), s, out[w0:w1])
    codec.finish()
    assert torch.equal(out, x)


def test_dtype_and_argument_errors(L):
    x = torch.zeros(100, dtype=torch.int32, device="cuda")
    o = torch.empty(10000, dtype=torch.uint8, device="cuda")
    with pytest.raises(L.LcfError) as e:
        L.lcf_compress("SPspeed", "float64", x, 400, o, 10000)
    assert e.value.status == 2
    with pytest.raises(L.LcfError) as e:
        L.lcf_compress("SPspeed", "float32", x, 402, o, 10000)
    assert e.value.status == 1
    with pytest.raises(L.LcfError) as e:
        L.lcf_compress("SPspeed", "float32", x, 400, o, 100)
    assert e.value.status == 3


def test_dpratio_decode_call_sizes(L, orc):
    """DPratio decodes of different sizes on one stream, chains in every one
    (the decoder's per-stream bitmaps and chain-node list must come back clean
    whatever the previous call's size was)."""
    rng = np.random.default_rng(11)
    base = rng.integers(0, 2**63, size=3000, dtype=np.uint64)
    for n in (60 * 2048 + 3, 5 * 2048, 90 * 2048 + 1000, 2048 + 7, 33 * 2048):
        w = np.resize(base[: 300 + n % 2000], n)
        w[n // 3: n // 3 + 500] = rng.integers(0, 2**63, size=500, dtype=np.uint64)  # a break in the chains
        check_parity(L, orc, "DPratio", w, f"size{n}")
