"""Seeded synthetic inputs shaped like the paper's workloads.

This module holds NO codec arithmetic: it only draws floating-point fields. It
is the one module both the oracle-side tests and the CUDA-side tests/bench use
(the GPU path never regenerates: parity tests copy the exact device bytes to the
host for the oracle).

Recipe: fields are smooth multi-scale sums of random-phase
cosines plus noise, computed in float64 with torch (on any device) and cast to
the codec's dtype. Seed = 0x4C4346 ^ (config_id << 32) ^ field_id.
PAPER.md L102: "scientific data that is relatively smooth ... normal, and
centered around zero"; L168: double-precision data has random low mantissa
bits (the σ noise term).
"""
from __future__ import annotations

import math

import numpy as np
import torch

# name -> (config_id, shape, dtype, {field_name: field_id})
CONFIGS = {
    "tiny_512x512_f32": (1, (512, 512), torch.float32, {"f": 0}),
    "cesm_1800x3600_f32": (2, (1800, 3600), torch.float32, {"T": 0, "U": 1}),
    "miranda_256x384x384_f64": (3, (256, 384, 384), torch.float64, {"density": 0, "velocity": 1, "rt_density": 2}),
    "nyx_512x512x512_f32": (4, (512, 512, 512), torch.float32, {"baryon_density": 0, "velocity": 1}),
    "hacc_280953867_f32": (5, (280_953_867,), torch.float32, {"xx": 0, "vx": 1}),
}


def seed_of(config_id: int, field_id: int) -> int:
    return (0x4C4346 ^ (config_id << 32) ^ field_id) & ((1 << 63) - 1)


def _gen(seed: int, device) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return g


def multiscale(shape, gen: torch.Generator, device, octaves: int = 6, waves: int = 8,
               dtype=torch.float64, origin=None, full_shape=None) -> torch.Tensor:
    """Σ_o 0.5^o · S_o(p), S_o = (1/√8) Σ_{8 waves} cos(2π k·p + φ), |k| ≈ 2·2^o.

    `origin`/`full_shape` let a caller draw a sub-block of a larger field (the
    same waves; sharded generation gives the same bytes as whole-field
    generation)."""
    full_shape = tuple(full_shape or shape)
    origin = tuple(origin or (0,) * len(shape))
    nd = len(shape)
    out = torch.zeros(shape, dtype=dtype, device=device)
    axes = []
    for d in range(nd):
        idx = torch.arange(origin[d], origin[d] + shape[d], dtype=dtype, device=device)
        axes.append(idx / full_shape[d])
    for o in range(octaves):
        mag = 2.0 * (2 ** o)
        dirs = torch.randn((waves, nd), generator=gen, device=device, dtype=torch.float64)
        dirs = dirs / dirs.norm(dim=1, keepdim=True).clamp_min(1e-12)
        ks = torch.round(dirs * mag)
        ks[ks.abs().sum(dim=1) == 0, 0] = 1.0
        phases = torch.rand((waves,), generator=gen, device=device, dtype=torch.float64) * 2 * math.pi
        acc = torch.zeros(shape, dtype=dtype, device=device)
        for w in range(waves):
            ph = torch.zeros(shape, dtype=dtype, device=device) + phases[w]
            for d in range(nd):
                view = [1] * nd
                view[d] = shape[d]
                ph = ph + (2 * math.pi * ks[w, d]) * axes[d].view(view)
            acc += torch.cos(ph)
        out += (0.5 ** o) * acc / math.sqrt(waves)
    return out


def field(config: str, name: str, device="cpu", origin=None, shape=None, replica: int = 0) -> torch.Tensor:
    """One synthetic field of a named config (optionally a sub-block);
    `replica` > 0 draws an independent field of the same kind (multi-GPU
    weak scaling concatenates replicas into one global stream)."""
    cid, full_shape, dtype, fields = CONFIGS[config]
    fid = fields[name]
    g = _gen(seed_of(cid, fid) ^ (replica << 20), device)
    shp = tuple(shape or full_shape)
    if config == "hacc_280953867_f32":
        return _hacc(name, g, device, shp, origin)
    ms = multiscale(shp, g, device, origin=origin, full_shape=full_shape)
    eps = torch.randn(shp, generator=g, device=device, dtype=torch.float64)
    if config == "tiny_512x512_f32":
        f = 0.0 + 1.0 * ms + 1e-3 * eps
    elif config == "cesm_1800x3600_f32":
        if name == "T":  # latitude-dominant temperature-like field
            lat = torch.linspace(-math.pi / 2, math.pi / 2, full_shape[0], dtype=torch.float64, device=device)
            o0 = (origin or (0, 0))[0]
            lat = lat[o0:o0 + shp[0]].view(-1, 1)
            f = 250.0 + 30.0 * (0.8 * torch.cos(lat) + 0.2 * ms) + 1e-4 * 30.0 * eps
        else:
            f = 0.0 + 20.0 * ms + 1e-3 * 20.0 * eps
    elif config == "miranda_256x384x384_f64":
        if name == "rt_density":
            return _rt_density(g, device, shp, origin, full_shape, ms, eps)
        if name == "density":
            fronts = torch.tanh(8.0 * multiscale(shp, g, device, octaves=2, origin=origin, full_shape=full_shape))
            f = 2.0 + (1.0 + fronts) * (0.5 + 0.5 * ms) + 1e-10 * eps
        else:
            f = 0.0 + 1.0 * ms + 1e-10 * eps
    elif config == "nyx_512x512x512_f32":
        if name == "baryon_density":
            f = torch.exp(1.5 * ms)
        else:
            f = 1e7 * ms + 1e-3 * 1e7 * eps
    else:
        raise KeyError(config)
    return f.to(dtype)


def _rt_density(g, device, shp, origin, full_shape, ms, eps):
    """Rayleigh–Taylor-like density (the flow Miranda simulates): a stratified
    background ρ0(z) along the fastest axis (z = last index / 384) plus a
    perturbation confined to a mixing band around z = 0.5 whose half-width
    δ(x, y) ∈ [0.12, 0.32] varies smoothly over the horizontal plane:
        f = ρ0(z) + w(x, y, z)·(0.3·ms + 1e-10·ε),
        ρ0(z) = 2 + tanh((z − 0.5)/0.08) + 0.25·z,
        w = max(0, 1 − ((z − 0.5)/δ)²)³.
    Outside the band w is exactly 0, so every (x, y) row repeats ρ0's bits
    there: the exact repeats at a distance of one row that FCM finds (L300,
    "repeating values … even when they are far apart"); about half the words
    match, and each match chains back through all earlier rows."""
    o = tuple(origin or (0, 0, 0))
    z = torch.arange(o[2], o[2] + shp[2], dtype=torch.float64, device=device) / full_shape[2]
    rho0 = 2.0 + torch.tanh((z - 0.5) / 0.08) + 0.25 * z  # a function of z alone: bitwise equal per row
    m2 = multiscale(shp[:2], g, device, octaves=3, origin=o[:2], full_shape=full_shape[:2])
    delta = (0.22 + 0.1 * torch.clamp(m2 / 1.5, -1.0, 1.0)).unsqueeze(-1)
    w = torch.clamp(1.0 - ((z - 0.5) / delta) ** 2, min=0.0) ** 3
    f = rho0 + w * (0.3 * ms + 1e-10 * eps)
    return f.to(torch.float64)


def _hacc(name, g, device, shp, origin):
    (n,) = shp
    if origin not in (None, (0,)):
        raise ValueError("HACC-like arrays are generated whole")
    if name == "xx":  # wrapped random walk of particle positions
        steps = torch.randn((n,), generator=g, device=device, dtype=torch.float64) * 0.01
        f = torch.remainder(torch.cumsum(steps, 0), 256.0)
    else:  # velocities: smoothed N(0, 300) + N(0, 30)
        base = torch.randn((n + 15,), generator=g, device=device, dtype=torch.float64) * 300.0
        c = torch.cumsum(base, 0)
        ma = (c[15:] - torch.cat([torch.zeros(1, dtype=c.dtype, device=device), c[:-16]])) / 16.0
        f = ma + torch.randn((n,), generator=g, device=device, dtype=torch.float64) * 30.0
    return f.to(torch.float32)


def smooth_1d(n: int, dtype=np.float32, seed: int = 0, sigma: float = 1e-3, scale: float = 1.0) -> np.ndarray:
    """Small host-side smooth series (random walk + noise) for unit tests."""
    rng = np.random.default_rng(seed)
    f = np.cumsum(rng.standard_normal(n)) * 0.01 * scale + sigma * rng.standard_normal(n)
    return f.astype(dtype)


# --- adversarial bit patterns --------------------------------------

F32_SPECIALS = np.array([
    0x00000000, 0x80000000, 0x7F800000, 0xFF800000,  # ±0, ±Inf
    0x7FC00000, 0x7FC00001, 0x7F800001, 0xFFBFFFFF,  # qNaN, qNaN payload, sNaN, -sNaN payload
    0x00000001, 0x007FFFFF, 0x3F800000, 0xBF800000,  # min/max denormal, ±1.0
    0x7F7FFFFF, 0xFF7FFFFF, 0x7FFFFFFF, 0x80000001,  # ±FLT_MAX, all-ones NaN, -min denormal
], dtype=np.uint32)

F64_SPECIALS = np.array([
    0x0000000000000000, 0x8000000000000000, 0x7FF0000000000000, 0xFFF0000000000000,
    0x7FF8000000000000, 0x7FF8000000000001, 0x7FF0000000000001, 0xFFF7FFFFFFFFFFFF,
    0x0000000000000001, 0x000FFFFFFFFFFFFF, 0x3FF0000000000000, 0xBFF0000000000000,
    0x7FEFFFFFFFFFFFFF, 0xFFEFFFFFFFFFFFFF, 0x7FFFFFFFFFFFFFFF, 0x8000000000000001,
], dtype=np.uint64)


def adversarial(word_bits: int, seed: int = 7):
    """List of (name, words) covering special values and pathological chunks."""
    rng = np.random.default_rng(seed)
    wdt = np.uint32 if word_bits == 32 else np.uint64
    fdt = np.float32 if word_bits == 32 else np.float64
    cw = 16384 * 8 // word_bits
    sp = F32_SPECIALS if word_bits == 32 else F64_SPECIALS
    out = []

    def rbits(n):
        return rng.integers(0, np.iinfo(wdt).max, size=n, dtype=wdt, endpoint=True)

    def smooth(n, s=0):
        return smooth_1d(n, fdt, seed=seed + s).view(wdt)

    out.append(("zeros", np.zeros(3 * cw + 5, dtype=wdt)))
    out.append(("constant_one", np.full(2 * cw + 77, sp[10], dtype=wdt)))
    out.append(("random_bits", rbits(2 * cw + 33)))
    out.append(("specials_cycle", np.resize(sp, 3 * cw + 19).astype(wdt)))
    out.append(("specials_random", sp[rng.integers(0, len(sp), size=2 * cw + 1)]))
    qnan, pmask = (wdt(0x7FC00000), wdt(0x003FFFFF)) if word_bits == 32 else \
        (wdt(0x7FF8000000000000), wdt(0x0007FFFFFFFFFFFF))
    out.append(("nan_payloads", (qnan | (rbits(cw + 9) & pmask)).astype(wdt)))
    out.append(("neg_zero_and_zero", np.where(rng.random(cw + 3) < 0.5, sp[0], sp[1]).astype(wdt)))
    out.append(("denormals", (rbits(cw + 100) & (sp[9])).astype(wdt)))
    out.append(("alt_sign", (smooth(2 * cw) ^ np.where(np.arange(2 * cw) % 2 == 1, sp[1], sp[0]).astype(wdt))))
    out.append(("max_min_pattern", np.resize(np.array([sp[14], sp[1]], dtype=wdt), 2 * cw + 31)))
    mixed = smooth(4 * cw, 1).copy()
    mixed[cw:2 * cw] = rbits(cw)  # incompressible chunk between smooth ones
    mixed[3 * cw:3 * cw + 100] = rbits(100)
    out.append(("mixed_incompressible", mixed))
    out.append(("smooth", smooth(5 * cw + 1035, 2)))
    out.append(("quantised", (np.round(smooth_1d(3 * cw, fdt, seed=seed) * 64) / 64).astype(fdt).view(wdt)))
    out.append(("repeats", np.repeat(smooth(3 * cw // 8 + 1, 3), 8)[: 3 * cw]))
    for n in (1, 2, 3, 31, 32, 33, 63, 64, 65, 127, 128, 129, cw - 1, cw, cw + 1, 3 * cw + 1035):
        out.append((f"tail_{n}", smooth(n, 4 + n)))
    return out


# --- every f32 bit pattern once -------------------------------------
# word i = P(i) for i in [0, 2^32), P the "lowbias32" integer mixer (xor-shift
# and odd-multiplier steps, each a bijection of u32): a seeded-looking order in
# which every 32-bit pattern appears exactly once. Host (numpy) and device
# (torch) give the same words.
_MIX = (16, 0x7FEB352D, 15, 0x846CA68B, 16)


def all_f32_patterns(start: int, count: int, device=None):
    """Words [start, start + count) of the permutation; numpy uint32 on the
    host (device None), else an int32 torch tensor on `device`."""
    if device is None:
        x = np.arange(start, start + count, dtype=np.uint64).astype(np.uint32)
        x ^= x >> np.uint32(_MIX[0])
        x *= np.uint32(_MIX[1])
        x ^= x >> np.uint32(_MIX[2])
        x *= np.uint32(_MIX[3])
        x ^= x >> np.uint32(_MIX[4])
        return x
    m = 0xFFFFFFFF
    x = torch.arange(start, start + count, dtype=torch.int64, device=device)
    x = x ^ (x >> _MIX[0])
    x = (x * _MIX[1]) & m
    x = x ^ (x >> _MIX[2])
    x = (x * _MIX[3]) & m
    x = x ^ (x >> _MIX[4])
    return x.to(torch.int32)  # wraps to the same 32 bits
