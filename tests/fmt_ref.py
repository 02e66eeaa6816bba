"""Independent, pure-Python readers of the LCF1 format (FORMAT.md).

Written from FORMAT.md alone (not from oracle/lcf_oracle.cpp) and used by the
oracle pin tests as a second formulation: a bit-order, field-order or offset
mistake in the oracle shows up as a disagreement here. Slow; small inputs only.
"""
from __future__ import annotations

import numpy as np


def ceil_div(a, b):
    return -(-a // b)


def round_up(a, b):
    return ceil_div(a, b) * b


def read_bits(buf: bytes, pos: int, w: int) -> int:
    """Field of width w at bit pos, LSB-first (FORMAT.md preamble)."""
    if w == 0:
        return 0
    as_int = int.from_bytes(buf, "little")
    return (as_int >> pos) & ((1 << w) - 1)


def zigzag(d: int, W: int) -> int:
    """Magnitude-sign of a signed d (L112/L126): 2d for d ≥ 0, −2d−1 otherwise."""
    return 2 * d if d >= 0 else -2 * d - 1


def unzigzag(u: int) -> int:
    return u // 2 if u % 2 == 0 else -(u + 1) // 2


def to_signed(v: int, W: int) -> int:
    v &= (1 << W) - 1
    return v - (1 << W) if v >> (W - 1) else v


def parse_mplg(buf: bytes, n: int, W: int):
    """Returns (list of (w, flag), field values before un-flagging, consumed)."""
    SW = 512 * 8 // W
    S = ceil_div(n, SW)
    off = round_up(S, 8)
    hdr, vals = [], []
    for s in range(S):
        ms = min(SW, n - s * SW)
        w, flag = buf[s] & 0x7F, buf[s] >> 7
        nb = ceil_div(ms * w, 8)
        seg = buf[off:off + nb]
        hdr.append((w, flag))
        vals.extend(read_bits(seg, j * w, w) for j in range(ms))
        off += nb
    return hdr, vals, off


def bitmap_bit(bm: bytes, j: int) -> int:
    return (bm[j // 8] >> (j % 8)) & 1


def unrepeat(buf: bytes, end: int, nxt: bytes, Lb: int):
    cnt = sum(bitmap_bit(nxt, j) for j in range(Lb))
    start = end - cnt
    assert start >= 0
    B, r, prev = bytearray(Lb), 0, 0
    for j in range(Lb):
        if bitmap_bit(nxt, j):
            prev = buf[start + r]
            r += 1
        B[j] = prev
    return bytes(B), start


def parse_rze(buf: bytes, L: int) -> bytes:
    L1 = ceil_div(L, 8)
    L2 = ceil_div(L1, 8)
    L3 = ceil_div(L2, 8)
    L4 = ceil_div(L3, 8)
    end = len(buf) - L4
    B4 = buf[end:]
    B3, end = unrepeat(buf, end, B4, L3)
    B2, end = unrepeat(buf, end, B3, L2)
    B1, end = unrepeat(buf, end, B2, L1)
    D, r = bytearray(L), 0
    for i in range(L):
        if bitmap_bit(B1, i):
            D[i] = buf[r]
            r += 1
    assert r == end, "nz(D) must end where nr(B1) starts"
    return bytes(D)


def rze_level_sizes(L: int):
    sizes = [L]
    for _ in range(4):
        sizes.append(ceil_div(sizes[-1], 8))
    return sizes  # bytes of D, B1, B2, B3, B4


def parse_adaptive(buf: bytes, rare: bool) -> bytes:
    L = buf[0] | (buf[1] << 8)
    k = buf[2]
    if k == 0:
        assert len(buf) == 3 + L
        return bytes(buf[3:])
    n, t = L // 8, L % 8
    L1 = ceil_div(n, 8)
    L2 = ceil_div(L1, 8)
    L3 = ceil_div(L2, 8)
    end = len(buf) - L3
    B3 = buf[end:]
    B2, end = unrepeat(buf, end, B3, L2)
    B1, end = unrepeat(buf, end, B2, L1)
    nset = sum(bitmap_bit(B1, i) for i in range(n))
    hib, lob = ceil_div(nset * k, 8), ceil_div(n * (64 - k), 8)
    assert 3 + hib + lob + t == end
    HI, LO = buf[3:3 + hib], buf[3 + hib:3 + hib + lob]
    out, hp, prev = bytearray(), 0, 0
    for i in range(n):
        if bitmap_bit(B1, i):
            top = read_bits(HI, hp * k, k)
            hp += 1
        else:
            top = prev if rare else 0
        prev = top
        low = read_bits(LO, i * (64 - k), 64 - k)
        out += ((top << (64 - k)) | low).to_bytes(8, "little")
    out += buf[3 + hib + lob:3 + hib + lob + t]
    return bytes(out)


def parse_stream(stream: bytes):
    """Header, table and per-chunk payload slices; asserts zero padding."""
    h = {
        "magic": int.from_bytes(stream[0:4], "little"),
        "version": stream[4], "algo": stream[5], "word_bytes": stream[6], "zero": stream[7],
        "n_bytes": int.from_bytes(stream[8:16], "little"),
        "n_chunks": int.from_bytes(stream[16:24], "little"),
        "payload_bytes": int.from_bytes(stream[24:32], "little"),
    }
    C = h["n_chunks"]
    table = [int.from_bytes(stream[32 + 4 * c:36 + 4 * c], "little") for c in range(C)]
    base = round_up(32 + 4 * C, 16)
    assert stream[32 + 4 * C:base] == bytes(base - 32 - 4 * C)
    chunks, off = [], base
    for e in table:
        ln, raw = e & 0x7FFFFFFF, e >> 31
        chunks.append((bool(raw), stream[off:off + ln]))
        assert stream[off + ln:off + round_up(ln, 16)] == bytes(round_up(ln, 16) - ln)
        off += round_up(ln, 16)
    assert off - base == h["payload_bytes"]
    assert len(stream) == off
    return h, table, chunks
