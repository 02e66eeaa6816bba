"""Pins of the CPU oracle against what PAPER.md and mathematics fix (-m "not gpu").

Each test names the passage (PAPER.md L<n>) or FORMAT.md reading it pins and is
chosen so that a plausible slip in oracle/lcf_oracle.cpp (dropped term, wrong
sign, index or bit order, transposed operand) fails it. Second formulations
live in tests/fmt_ref.py and in this file; none calls oracle code to compute
an expected value.
"""
import itertools

import numpy as np
import pytest

import fmt_ref
from conftest import golden_lines
from paper_conf_asplos_azamifb25_b200 import datagen

U32, U64 = np.uint32, np.uint64


# ---- DIFFMS / TCMS (L110–112, Fig. 2 caption L126) --------------------------

def test_tcms_is_textbook_zigzag(orc):
    """Golden zigzag table; DIFFMS of a single word is TCMS(x − 0) (L112)."""
    for d, u in golden_lines("zigzag.txt"):
        d, u = int(d), int(u)
        got32 = orc.diffms_enc(np.array([d & 0xFFFFFFFF], dtype=U32))[0]
        got64 = orc.diffms_enc(np.array([d & (2**64 - 1)], dtype=U64))[0]
        assert int(got32) == u and int(got64) == u


def test_diffms_hand_vector(orc):
    """1.0f, next float up, next float down: x0 kept vs 0, then +1, −2 (L112)."""
    x = np.array([0x3F800000, 0x3F800001, 0x3F7FFFFF], dtype=U32)
    assert orc.diffms_enc(x).tolist() == [0x7F000000, 2, 3]


@pytest.mark.parametrize("W", [32, 64])
def test_diffms_matches_magnitude_sign_definition(orc, W):
    """u[i] = magnitude-sign(x[i] − x[i−1] mod 2^W as signed), arithmetic form."""
    rng = np.random.default_rng(W)
    dt = U32 if W == 32 else U64
    x = rng.integers(0, 2**W - 1, size=300, dtype=dt, endpoint=True)
    x[100:200] = (np.arange(100) * 3).astype(dt)  # small differences too
    u = orc.diffms_enc(x)
    prev = 0
    for i in range(len(x)):
        d = fmt_ref.to_signed(int(x[i]) - prev, W)
        assert int(u[i]) == fmt_ref.zigzag(d, W), i
        prev = int(x[i])


@pytest.mark.parametrize("W", [32, 64])
def test_diffms_decode_is_wrapping_cumsum(orc, W):
    rng = np.random.default_rng(3 + W)
    dt = U32 if W == 32 else U64
    u = rng.integers(0, 2**W - 1, size=1000, dtype=dt, endpoint=True)
    d = np.array([fmt_ref.unzigzag(int(v)) % 2**W for v in u], dtype=dt)
    expect = np.cumsum(d, dtype=dt)  # numpy unsigned cumsum wraps mod 2^W
    assert np.array_equal(orc.diffms_dec(u), expect)
    assert np.array_equal(orc.diffms_enc(orc.diffms_dec(u)), u)


# ---- MPLG (L114–118, Fig. 3 caption L130) ------------------------------------

def test_mplg_figure3_example(orc):
    g = dict((k, int(v)) for k, v in golden_lines("mplg_fig3.txt"))
    v0 = (1 << (32 - g["leading_zeros_of_max"] - 1)) | 0x2BCDE  # max, 12 leading zeros
    vals = [v0, 0x123, 0x12345]
    enc = orc.mplg_enc(np.array(vals, dtype=U32))
    assert enc[0] == g["kept_bits"] and enc[1:8] == bytes(7)  # header, padded to 8
    packed = sum(v << (g["kept_bits"] * j) for j, v in enumerate(vals))
    assert enc[8:] == packed.to_bytes(-(-g["concatenated_bits"] // 8), "little")


@pytest.mark.parametrize("W", [32, 64])
def test_mplg_brute_force_width_and_flag(orc, W):
    """w = minimal width holding every value; flag iff max has no leading zero."""
    rng = np.random.default_rng(11 + W)
    dt = U32 if W == 32 else U64
    SW = 4096 // W
    n = 5 * SW + 7
    u = np.zeros(n, dtype=dt)
    widths = []
    for s in range(6):
        w = int(rng.integers(0, W + 1))
        widths.append(w)
        m = min(SW, n - s * SW)
        vals = rng.integers(0, 2**W - 1, size=m, dtype=dt, endpoint=True)
        u[s * SW:s * SW + m] = vals & dt((1 << w) - 1) if w < W else vals
    enc = orc.mplg_enc(u)
    hdr, fields, consumed = fmt_ref.parse_mplg(enc, n, W)
    assert consumed == len(enc)
    for s, (w, flag) in enumerate(hdr):
        sub = [int(v) for v in u[s * SW:(s + 1) * SW]]
        expect_flag = int(max(sub) >> (W - 1) == 1)
        vals = [fmt_ref.zigzag(fmt_ref.to_signed(v, W), W) for v in sub] if expect_flag else sub
        expect_w = next(b for b in range(W + 1) if all(v < (1 << b) for v in vals))
        assert (w, flag) == (expect_w, expect_flag)
        assert fields[s * SW:s * SW + len(sub)] == vals
    assert np.array_equal(orc.mplg_dec(enc, n, dt), u)


def test_mplg_closed_forms_through_streams(orc):
    """All-zero SP chunk: 32 header bytes only; constant 1.0f: 32 + 16·31 = 528
    (only word 0 is non-zero, zz(0x3F800000) = 0x7F000000 has 31 bits); DP
    analogues 32 and 32 + 8·63 = 536."""
    for algo, arr, expect in [
        ("SPspeed", np.zeros(4096, np.float32), 32),
        ("SPspeed", np.ones(4096, np.float32), 528),
        ("DPspeed", np.zeros(2048, np.float64), 32),
        ("DPspeed", np.ones(2048, np.float64), 536),
    ]:
        h, table, chunks = fmt_ref.parse_stream(orc.compress(algo, arr))
        assert table == [expect]


# ---- BIT (L140–142, Fig. 4 caption L152, L162) -------------------------------

def test_bit_transpose_against_unpackbits(orc):
    rng = np.random.default_rng(5)
    for m in (32, 64, 100, 4096, 4095):
        u = rng.integers(0, 2**32 - 1, size=m, dtype=U32, endpoint=True)
        T = orc.bit32_enc(u)
        G = m // 32
        # bits[g, i, b] = bit b (MSB first) of word 32g+i
        bits = np.unpackbits(u[:32 * G].astype(">u4").view(np.uint8)).reshape(G, 32, 32)
        planes = bits.transpose(2, 0, 1)  # [p, g, i]; p = 0 is the MSB plane
        expect = (planes.astype(np.uint64) << np.arange(32, dtype=np.uint64)).sum(axis=2).astype(U32)
        assert np.array_equal(T[:32 * G].reshape(32, G), expect)
        assert np.array_equal(T[32 * G:], u[32 * G:])
        assert np.array_equal(orc.bit32_dec(T), u)
        assert sum(bin(int(v)).count("1") for v in T) == sum(bin(int(v)).count("1") for v in u)


def test_bit_small_leading_zero_values_give_zero_leading_planes(orc):
    """L142: values with many leading zeros → the first planes are all zero."""
    u = np.arange(4096, dtype=U32) % 1000  # < 2^10
    T = orc.bit32_enc(u)
    assert not T[: 22 * 128].any() and T[22 * 128:].any()


# ---- RZE (L144–148, L158) ------------------------------------------------------

def test_rze_level_sizes_match_paper():
    (rze_bits,) = [list(map(int, r[1:])) for r in golden_lines("rze_levels.txt") if r[0] == "rze_bits"]
    sizes = fmt_ref.rze_level_sizes(16384)
    assert [8 * s for s in sizes[1:]] == rze_bits


@pytest.mark.parametrize("case", ["zeros", "sparse", "dense", "ragged"])
def test_rze_closed_form_and_independent_parse(orc, case):
    rng = np.random.default_rng(17)
    L = 16384 if case != "ragged" else 4 * 1035
    if case == "zeros":
        D = np.zeros(L, np.uint8)
    elif case == "sparse":
        D = (rng.random(L) < 0.05).astype(np.uint8) * rng.integers(1, 256, L).astype(np.uint8)
        D[:8000] = 0
    else:
        D = rng.integers(0, 256, L).astype(np.uint8)
        D[rng.random(L) < 0.3] = 0
    enc = orc.rze_enc(D)
    # closed form: |nz(D)| + Σ_levels |non-repeating bytes| + |B4|
    sizes = fmt_ref.rze_level_sizes(L)
    B = np.zeros(sizes[1], np.uint8)
    nzb = np.flatnonzero(D)
    np.bitwise_or.at(B, nzb // 8, (1 << (nzb % 8)).astype(np.uint8))
    total = len(nzb)
    for _lvl in range(3):
        prev = np.concatenate([[0], B[:-1]]).astype(np.uint8)
        diff = B != prev
        total += int(diff.sum())
        nxt = np.zeros(-(-len(B) // 8), np.uint8)
        idx = np.flatnonzero(diff)
        np.bitwise_or.at(nxt, idx // 8, (1 << (idx % 8)).astype(np.uint8))
        B = nxt
    total += len(B)
    assert len(enc) == total
    if case == "zeros":
        assert len(enc) == 4  # only the 32-bit B4 remains
    assert fmt_ref.parse_rze(enc, L) == D.tobytes()
    assert orc.rze_dec(enc, L) == D.tobytes()


# ---- FCM (L170–185, Fig. 6; decode L197) ----------------------------------------

def test_fcm_figure6_exact(orc):
    rows = {r[0]: r[1:] for r in golden_lines("fig6_fcm.txt")}
    sym = {"a": 0x400921FB54442D18, "b": 0xC00921FB54442D18, "c": 0x7FF8000000000001, "0": 0}
    x = np.array([sym[s] for s in rows["value"]], dtype=U64)
    h = np.array([int(v) for v in rows["hash"]], dtype=U32)
    V, D = orc.fcm_match(x, h)
    assert V.tolist() == [sym[s] for s in rows["V"]]
    assert D.tolist() == [int(v) for v in rows["Dist"]]
    assert np.array_equal(orc.fcm_dec(V, D), x)


def test_fcm_match_equals_recency_table(orc):
    """Sorted-pair formulation == "nearest of the 4 most recent same-hash
    predecessors with the same value" (a per-hash recency list)."""
    rng = np.random.default_rng(23)
    for trial in range(20):
        n = int(rng.integers(1, 400))
        x = rng.integers(0, 4, n).astype(U64) * U64(0x3FF0000000000001)
        h = rng.integers(0, int(rng.integers(1, 6)), n).astype(U32)
        V, D = orc.fcm_match(x, h)
        recent = {}
        for i in range(n):
            lst = recent.setdefault(int(h[i]), [])
            dist = 0
            for j in reversed(lst[-4:]):
                if x[j] == x[i]:
                    dist = i - j
                    break
            assert int(D[i]) == dist and int(V[i]) == (0 if dist else int(x[i])), (trial, i)
            lst.append(i)


def test_fcm_hash_definition_and_invariants(orc):
    x = datagen.smooth_1d(5000, np.float64, seed=2).view(U64)
    x[1000:1100] = x[900:1000]  # exact repeats
    h = orc.fcm_hash(x)
    assert int(h.max()) < 2**20
    K1, K2, K3 = 0x9E3779B97F4A7C15, 0xC2B2AE3D27D4EB4F, 0x165667B19E3779F9
    for i in (0, 1, 2, 3, 1234):
        a, b, c = [int(x[i - k]) if i - k >= 0 else 0 for k in (1, 2, 3)]
        assert int(h[i]) == (((a * K1) ^ (b * K2) ^ (c * K3)) % 2**64) >> 44
    V, D = orc.fcm_match(x, h)
    idx = np.flatnonzero(D)
    assert len(idx) >= 90
    assert np.all(D[idx] <= idx) and not V[idx].any()
    assert np.array_equal(x[idx - D[idx].astype(np.int64)], x[idx])
    assert np.array_equal(orc.fcm_dec(V, D), x)


def test_fcm_decode_rejects_forward_distance(orc):
    with pytest.raises(orc.OracleError):
        orc.fcm_dec(np.zeros(3, U64), np.array([0, 2, 0], dtype=U64))


# ---- RAZE / RARE (L189, Fig. 7) -------------------------------------

def _exact_bits(words, k, rare):
    prev, nset = 0, 0
    for v in words:
        top = v >> (64 - k)
        if top != ((prev >> (64 - k)) if rare else 0):
            nset += 1
        prev = v
    return nset * k + len(words) * (64 - k)


@pytest.mark.parametrize("rare", [False, True])
@pytest.mark.parametrize("kind", ["smooth", "quantised", "zeros", "small", "random"])
def test_adaptive_k_is_brute_force_optimum(orc, rare, kind):
    rng = np.random.default_rng(31)
    n = 2048 if kind != "small" else 37
    if kind == "smooth":
        w = orc.diffms_enc(datagen.smooth_1d(n, np.float64, seed=4).view(U64))
    elif kind == "quantised":
        w = orc.diffms_enc((np.round(datagen.smooth_1d(n, np.float64, seed=5) * 16) / 16).view(U64))
    elif kind == "zeros":
        w = np.zeros(n, U64)
    elif kind == "small":
        w = rng.integers(0, 2**20, n).astype(U64)
    else:
        w = rng.integers(0, 2**64 - 1, n, dtype=U64, endpoint=True)
    data = w.tobytes() + b"\x05\x06\x07"  # 3 tail bytes
    enc = (orc.rare_enc if rare else orc.raze_enc)(data)
    L = len(data)
    assert enc[0] | (enc[1] << 8) == L
    words = [int(v) for v in w]
    costs = {k: _exact_bits(words, k, rare) for k in range(1, 65)}
    kstar = min(costs, key=lambda k: (costs[k], k))
    if enc[2] == 0:
        assert len(enc) == 3 + L and enc[3:] == data  # bypass (A-23)
    else:
        assert enc[2] == kstar
        if kind == "zeros":
            assert kstar == 64 and len(enc) == 3 + 0 + 0 + 3 + 0 + 0 + 4
    assert fmt_ref.parse_adaptive(enc, rare) == data
    assert (orc.rare_dec if rare else orc.raze_dec)(enc) == data
    if kind == "random":
        assert enc[2] == 0


def test_raze_level_sizes_match_paper():
    (bits,) = [list(map(int, r[1:])) for r in golden_lines("rze_levels.txt") if r[0] == "raze_bits"]
    n = 2048
    L1 = -(-n // 8)
    L2 = -(-L1 // 8)
    L3 = -(-L2 // 8)
    assert [n, 8 * L2, 8 * L3] == bits


# ---- whole streams ----------------------------------------------------------------

ALGOS = ["SPspeed", "SPratio", "DPspeed", "DPratio"]


@pytest.mark.parametrize("algo", ALGOS)
def test_stream_roundtrip_adversarial(orc, algo):
    W = 32 if algo.startswith("SP") else 64
    for name, words in datagen.adversarial(W):
        s = orc.compress(algo, words)
        h, table, chunks = fmt_ref.parse_stream(s)
        assert h["magic"] == 0x3146434C and h["version"] == 1 and h["algo"] == ALGOS.index(algo)
        assert h["n_bytes"] == words.nbytes
        raw_len = 16384
        for c, (raw, pay) in enumerate(chunks):
            if raw:
                assert pay in (words.tobytes()[c * raw_len:(c + 1) * raw_len],) or algo == "DPratio"
        out = orc.decompress(algo, s)
        assert np.array_equal(out, words), name
        assert orc.compress(algo, words) == s  # deterministic (L415)


@pytest.mark.parametrize("algo", ALGOS)
def test_exhaustive_tiny_streams(orc, algo):
    """Every 1-, 2- and 3-word stream over a 16-value special alphabet."""
    sp = datagen.F32_SPECIALS if algo.startswith("SP") else datagen.F64_SPECIALS
    for r in (1, 2, 3):
        for combo in itertools.product(range(16), repeat=r):
            words = sp[list(combo)]
            s = orc.compress(algo, words)
            assert np.array_equal(orc.decompress(algo, s), words)


def test_empty_input(orc):
    for algo in ALGOS:
        s = orc.compress(algo, np.zeros(0, np.uint8))
        assert len(s) == 32
        assert orc.decompress(algo, s).size == 0


def test_speed_codec_mplg_payload_parses(orc):
    """Chunk payloads of SPspeed are MPLG over DIFFMS (L350), parsed independently."""
    x = datagen.smooth_1d(3 * 4096 + 1035, np.float32, seed=9).view(U32)
    _, table, chunks = fmt_ref.parse_stream(orc.compress("SPspeed", x))
    for c, (raw, pay) in enumerate(chunks):
        xs = x[c * 4096:(c + 1) * 4096]
        _, fields, consumed = fmt_ref.parse_mplg(pay, len(xs), 32)
        assert consumed == len(pay)
        prev, rec = 0, []
        hdr, _, _ = fmt_ref.parse_mplg(pay, len(xs), 32)
        for j, v in enumerate(fields):
            flag = hdr[j // 128][1]
            d = fmt_ref.unzigzag(fmt_ref.unzigzag(v) % 2**32) if flag else fmt_ref.unzigzag(v)
            prev = (prev + d) % 2**32
            rec.append(prev)
        assert rec == xs.tolist()


def test_spratio_and_dpratio_payloads_parse(orc):
    x = datagen.smooth_1d(4096 + 100, np.float32, seed=12).view(U32)
    _, _, chunks = fmt_ref.parse_stream(orc.compress("SPratio", x))
    for c, (raw, pay) in enumerate(chunks):
        m = len(x[c * 4096:(c + 1) * 4096])
        assert not raw
        D = np.frombuffer(fmt_ref.parse_rze(pay, 4 * m), U32)
        assert np.array_equal(orc.diffms_dec(orc.bit32_dec(D)), x[c * 4096:c * 4096 + m])
    y = datagen.smooth_1d(2048 + 50, np.float64, seed=13).view(U64)
    y[100:150] = y[10:60]
    _, _, chunks = fmt_ref.parse_stream(orc.compress("DPratio", y))
    assert len(chunks) == 4
    V, D = orc.fcm_match(y, orc.fcm_hash(y))
    for c, (raw, pay) in enumerate(chunks):
        arr = V if c % 2 == 0 else D
        t = c // 2
        part = arr[t * 2048:(t + 1) * 2048]
        if raw:
            assert pay == part.tobytes()
            continue
        inner = fmt_ref.parse_adaptive(fmt_ref.parse_adaptive(pay, True), False)
        assert np.array_equal(orc.diffms_dec(np.frombuffer(inner, U64)), part)


def test_compress_chunks_slices_equal_full_stream(orc):
    x = datagen.smooth_1d(7 * 4096 + 333, np.float32, seed=21).view(U32)
    full = orc.compress("SPspeed", x)
    h, table, chunks = fmt_ref.parse_stream(full)
    base = fmt_ref.round_up(32 + 4 * len(table), 16)
    for first, cnt in [(0, 3), (3, 5), (0, 8), (7, 1)]:
        tab, pay = orc.compress_chunks("SPspeed", x, first, cnt)
        assert tab.tolist() == table[first:first + cnt]
        start = base + sum(fmt_ref.round_up(e & 0x7FFFFFFF, 16) for e in table[:first])
        assert pay == full[start:start + len(pay)]


def test_corrupt_headers_are_rejected(orc):
    x = datagen.smooth_1d(3 * 4096, np.float32, seed=1)
    s = bytearray(orc.compress("SPspeed", x))
    assert orc.decompress_status("SPratio", bytes(s)) == 2  # dtype/algo mismatch
    for off, val in [(0, 0x00), (4, 2), (6, 8), (16, 9), (24, 0xFF), (32, 0xFF), (35, 0x7F)]:
        t = bytearray(s)
        t[off] = val
        assert orc.decompress_status("SPspeed", bytes(t)) == 4, off
    assert orc.decompress_status("SPspeed", bytes(s[:-16])) == 4
    assert orc.decompress_status("SPspeed", bytes(s), out_capacity=100) == 3
    rng = np.random.default_rng(0)
    for _ in range(200):  # random garbage in table/payload: reject or decode, never crash
        t = bytearray(s)
        pos = int(rng.integers(32, len(t)))
        t[pos] = int(rng.integers(0, 256))
        orc.decompress_status("SPspeed", bytes(t))
