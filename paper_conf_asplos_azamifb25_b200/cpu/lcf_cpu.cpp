// lcf_cpu.cpp — the multi-threaded CPU codec: the four
// codecs of PAPER.md §3 (L104–201) over the LCF1 stream of FORMAT.md, with the
// paper's CPU parallelisation (L104, L120). Written from FORMAT.md; it shares
// no code with the oracle (oracle/) or the B200 kernels (csrc/). Stage codecs
// work on whole words (32/64-bit accumulators, a 32×32 bit-matrix transpose),
// not bit by bit.
#include "lcf_cpu.h"

#include <algorithm>
#include <atomic>
#include <cstring>
#include <memory>
#include <new>
#include <thread>
#include <vector>

namespace {

enum : int { kOk = 0, kInvalid = 1, kDtype = 2, kSmall = 3, kCorrupt = 4, kOom = 6 };
constexpr size_t kChunkBytes = 16384, kHeader = 32;
constexpr uint32_t kMagic = 0x3146434Cu, kRawFlag = 0x80000000u;
constexpr uint32_t kTile = 2048;  // DPratio tile (= DP chunk words)
constexpr size_t kBuf = 2 * kChunkBytes + 256;  // per-thread stage buffers

inline size_t r16(size_t x) { return (x + 15) & ~size_t(15); }
inline size_t cdiv(size_t a, size_t b) { return (a + b - 1) / b; }
inline uint32_t ld32(const uint8_t* p) { uint32_t v; std::memcpy(&v, p, 4); return v; }
inline uint64_t ld64(const uint8_t* p) { uint64_t v; std::memcpy(&v, p, 8); return v; }
inline void st32(uint8_t* p, uint32_t v) { std::memcpy(p, &v, 4); }
inline void st64(uint8_t* p, uint64_t v) { std::memcpy(p, &v, 8); }

int word_bytes(int algo) { return (algo == 0 || algo == 1) ? 4 : (algo == 2 || algo == 3) ? 8 : 0; }
bool dtype_ok(int algo, int dtype) { return dtype == (word_bytes(algo) == 8 ? 1 : 0); }

// ---- FORMAT.md notation: zz / unzz (L112), clz, bitlen ----
inline uint32_t zz(uint32_t d) { return (d << 1) ^ (uint32_t)((int32_t)d >> 31); }
inline uint64_t zz(uint64_t d) { return (d << 1) ^ (uint64_t)((int64_t)d >> 63); }
inline uint32_t unzz(uint32_t u) { return (u >> 1) ^ (0u - (u & 1u)); }
inline uint64_t unzz(uint64_t u) { return (u >> 1) ^ (0ull - (u & 1ull)); }
inline uint32_t clz(uint32_t v) { return v ? (uint32_t)__builtin_clz(v) : 32u; }
inline uint32_t clz(uint64_t v) { return v ? (uint32_t)__builtin_clzll(v) : 64u; }
template <class T> inline uint32_t bitlen(T v) { return 8 * sizeof(T) - clz(v); }

// ---- LSB-first bit streams (FORMAT.md preamble) ----
struct BitW {  // writes whole 32-bit words; finish() writes the last partial bytes
  uint8_t* p;
  size_t pos = 0;  // bytes written
  uint64_t acc = 0;
  uint32_t nb = 0;  // pending bits (< 32)
  explicit BitW(uint8_t* out) : p(out) {}
  void put32(uint32_t v, uint32_t w) {  // v < 2^w, w ≤ 32
    acc |= (uint64_t)v << nb;
    nb += w;
    if (nb >= 32) {
      st32(p + pos, (uint32_t)acc);
      pos += 4;
      acc >>= 32;
      nb -= 32;
    }
  }
  void put(uint64_t v, uint32_t w) {  // v < 2^w, w ≤ 64
    if (w > 32) {
      put32((uint32_t)v, 32);
      put32((uint32_t)(v >> 32), w - 32);
    } else if (w) {
      put32((uint32_t)v, w);
    }
  }
  size_t finish() {
    for (; nb > 0; nb = nb > 8 ? nb - 8 : 0) {
      p[pos++] = (uint8_t)acc;
      acc >>= 8;
    }
    return pos;
  }
};
struct BitR {  // reads fields at increasing bit positions; needs 8 readable bytes of slack
  const uint8_t* p;
  uint64_t bit = 0;
  explicit BitR(const uint8_t* in) : p(in) {}
  uint32_t get32(uint32_t w) {  // w ≤ 32
    if (!w) return 0;
    const uint64_t v = ld64(p + (bit >> 3)) >> (bit & 7);
    bit += w;
    return w == 32 ? (uint32_t)v : (uint32_t)v & ((1u << w) - 1u);
  }
  uint64_t get(uint32_t w) {  // w ≤ 64
    if (w > 32) {
      const uint64_t lo = get32(32);
      return lo | ((uint64_t)get32(w - 32) << 32);
    }
    return get32(w);
  }
};

// ---- DIFFMS_W (FORMAT.md §3) ----
template <class T> void diffms(const T* x, T* u, size_t m) {
  T prev = 0;
  for (size_t i = 0; i < m; ++i) {
    u[i] = zz((T)(x[i] - prev));
    prev = x[i];
  }
}
template <class T> void undiffms(T* u, size_t m) {
  T acc = 0;
  for (size_t i = 0; i < m; ++i) {
    acc = (T)(acc + unzz(u[i]));
    u[i] = acc;
  }
}

// ---- MPLG_W (FORMAT.md §4): 512-byte subchunks ----
template <class T> size_t mplg_enc(const T* u, size_t m, uint8_t* out) {
  constexpr size_t SW = 512 / sizeof(T);
  constexpr uint32_t W = 8 * sizeof(T);
  const size_t S = cdiv(m, SW), hdr = (S + 7) & ~size_t(7);
  std::memset(out, 0, hdr);
  size_t pos = hdr;
  T v[SW];
  for (size_t s = 0; s < S; ++s) {
    const size_t ms = std::min(SW, m - s * SW);
    T mx = 0;
    for (size_t j = 0; j < ms; ++j) mx = std::max(mx, u[s * SW + j]);
    const bool flag = (mx >> (W - 1)) != 0;  // the "enhanced" TCMS retry (L114)
    mx = 0;
    for (size_t j = 0; j < ms; ++j) {
      v[j] = flag ? zz(u[s * SW + j]) : u[s * SW + j];
      mx = std::max(mx, v[j]);
    }
    const uint32_t w = bitlen(mx);
    out[s] = (uint8_t)(w | (flag ? 0x80u : 0u));
    BitW bw(out + pos);
    for (size_t j = 0; j < ms; ++j) bw.put(v[j], w);
    pos += bw.finish();
  }
  return pos;
}
// in: len bytes with ≥ 8 readable bytes of slack. Returns false if malformed.
template <class T> bool mplg_dec(const uint8_t* in, size_t len, T* u, size_t m) {
  constexpr size_t SW = 512 / sizeof(T);
  constexpr uint32_t W = 8 * sizeof(T);
  const size_t S = cdiv(m, SW), hdr = (S + 7) & ~size_t(7);
  if (len < hdr) return false;
  size_t total = hdr;
  for (size_t s = 0; s < S; ++s) {
    const uint32_t w = in[s] & 127u;
    if (w > W) return false;
    total += cdiv(std::min(SW, m - s * SW) * w, 8);
  }
  if (total != len) return false;
  size_t pos = hdr;
  for (size_t s = 0; s < S; ++s) {
    const size_t ms = std::min(SW, m - s * SW);
    const uint32_t w = in[s] & 127u;
    const bool flag = in[s] >> 7;
    BitR br(in + pos);
    for (size_t j = 0; j < ms; ++j) {
      const T f = (T)br.get(w);
      u[s * SW + j] = flag ? unzz(f) : f;
    }
    pos += cdiv(ms * w, 8);
  }
  undiffms(u, m);
  return true;
}

// ---- BIT₃₂ (FORMAT.md §5.1) ----
// In-place 32×32 transpose: afterwards bit i of a[b] = old bit b of a[i].
void transpose32(uint32_t a[32]) {
  uint32_t msk = 0x0000FFFFu;
  for (uint32_t j = 16; j; j >>= 1, msk ^= msk << j) {
    for (uint32_t k = 0; k < 32; k = ((k | j) + 1) & ~j) {
      const uint32_t t = ((a[k] >> j) ^ a[k | j]) & msk;
      a[k] ^= t << j;
      a[k | j] ^= t;
    }
  }
}
void bit_enc(const uint32_t* u, size_t m, uint32_t* T) {
  const size_t G = m / 32;
  uint32_t a[32];
  for (size_t g = 0; g < G; ++g) {
    std::memcpy(a, u + 32 * g, sizeof a);
    transpose32(a);
    for (uint32_t p = 0; p < 32; ++p) T[p * G + g] = a[31 - p];  // MSB plane first (A-9)
  }
  for (size_t i = 32 * G; i < m; ++i) T[i] = u[i];
}
void bit_dec(const uint32_t* T, size_t m, uint32_t* u) {
  const size_t G = m / 32;
  uint32_t a[32];
  for (size_t g = 0; g < G; ++g) {
    for (uint32_t p = 0; p < 32; ++p) a[31 - p] = T[p * G + g];
    transpose32(a);
    std::memcpy(u + 32 * g, a, sizeof a);
  }
  for (size_t i = 32 * G; i < m; ++i) u[i] = T[i];
}

// ---- repetition elimination of a bitmap (L146): B_{l+1} bit j = [B_l[j] ≠ B_l[j−1]] ----
void rep_bits(const uint8_t* B, size_t Ln, uint8_t* Bn) {
  std::memset(Bn, 0, cdiv(Ln, 8));
  uint8_t prev = 0;
  for (size_t j = 0; j < Ln; ++j) {
    if (B[j] != prev) Bn[j >> 3] |= (uint8_t)(1u << (j & 7));
    prev = B[j];
  }
}
size_t put_nr(const uint8_t* B, size_t Ln, const uint8_t* Bn, uint8_t* out) {  // nr(B_l)
  size_t o = 0;
  for (size_t j = 0; j < Ln; ++j)
    if ((Bn[j >> 3] >> (j & 7)) & 1) out[o++] = B[j];
  return o;
}
size_t popc_bits(const uint8_t* B, size_t nbits) {  // set bits among the first nbits
  size_t c = 0, j = 0;
  for (; j + 64 <= nbits; j += 64) c += (size_t)__builtin_popcountll(ld64(B + j / 8));
  for (; j + 8 <= nbits; j += 8) c += (size_t)__builtin_popcount(B[j / 8]);
  if (j < nbits) c += (size_t)__builtin_popcount(B[j / 8] & ((1u << (nbits - j)) - 1u));
  return c;
}
// B_l (Ln bytes) from B_{l+1} and the nr(B_l) bytes at src (count popc(B_{l+1} bits < Ln)).
void get_nr(const uint8_t* src, const uint8_t* Bn, size_t Ln, uint8_t* B) {
  size_t r = 0;
  for (size_t j = 0; j < Ln; ++j) {
    r += (Bn[j >> 3] >> (j & 7)) & 1;
    B[j] = r ? src[r - 1] : 0;
  }
}

// ---- RZE (FORMAT.md §5.2) ----
size_t rze_enc(const uint8_t* D, size_t L, uint8_t* out) {
  const size_t L1 = cdiv(L, 8), L2 = cdiv(L1, 8), L3 = cdiv(L2, 8), L4 = cdiv(L3, 8);
  uint8_t B1[kChunkBytes / 8], B2[kChunkBytes / 64 + 1], B3[kChunkBytes / 512 + 1], B4[8];
  std::memset(B1, 0, L1);
  size_t o = 0;
  for (size_t q = 0; q < L1; ++q) {
    const size_t i0 = 8 * q, e = std::min<size_t>(8, L - i0);
    if (e == 8 && ld64(D + i0) == 0) continue;
    uint32_t b = 0;
    for (size_t i = 0; i < e; ++i)
      if (D[i0 + i]) {
        b |= 1u << i;
        out[o++] = D[i0 + i];
      }
    B1[q] = (uint8_t)b;
  }
  rep_bits(B1, L1, B2);
  rep_bits(B2, L2, B3);
  rep_bits(B3, L3, B4);
  o += put_nr(B1, L1, B2, out + o);
  o += put_nr(B2, L2, B3, out + o);
  o += put_nr(B3, L3, B4, out + o);
  std::memcpy(out + o, B4, L4);
  return o + L4;
}
bool rze_dec(const uint8_t* in, size_t len, uint8_t* D, size_t L) {
  const size_t L1 = cdiv(L, 8), L2 = cdiv(L1, 8), L3 = cdiv(L2, 8), L4 = cdiv(L3, 8);
  uint8_t B1[kChunkBytes / 8], B2[kChunkBytes / 64 + 1], B3[kChunkBytes / 512 + 1];
  if (len < L4) return false;
  const uint8_t* B4 = in + len - L4;
  const size_t c3 = popc_bits(B4, L3);
  if (len - L4 < c3) return false;
  const size_t s3 = len - L4 - c3;
  get_nr(in + s3, B4, L3, B3);
  const size_t c2 = popc_bits(B3, L2);
  if (s3 < c2) return false;
  const size_t s2 = s3 - c2;
  get_nr(in + s2, B3, L2, B2);
  const size_t c1 = popc_bits(B2, L1);
  if (s2 < c1) return false;
  const size_t s1 = s2 - c1;
  get_nr(in + s1, B2, L1, B1);
  if (popc_bits(B1, L) != s1) return false;
  size_t r = 0;
  for (size_t q = 0; q < L1; ++q) {
    const uint32_t b = B1[q];
    const size_t i0 = 8 * q, e = std::min<size_t>(8, L - i0);
    if (!b) {
      std::memset(D + i0, 0, e);
      continue;
    }
    for (size_t i = 0; i < e; ++i) D[i0 + i] = ((b >> i) & 1) ? in[r++] : 0;
  }
  return true;
}

// ---- RAZE / RARE (FORMAT.md §6.2–6.3) ----
size_t adaptive_enc(const uint8_t* in, size_t L, uint8_t* out, bool rare) {
  const size_t n = L / 8, t = L % 8;  // n ≤ 2048 (L ≤ 3 + 16384)
  uint64_t v[kChunkBytes / 8 + 1];
  uint32_t cnt[65] = {0};
  for (size_t i = 0; i < n; ++i) {
    v[i] = ld64(in + 8 * i);
    cnt[clz((uint64_t)(v[i] ^ (rare && i ? v[i - 1] : (uint64_t)0)))]++;
  }
  uint32_t k = 1;  // smallest argmin of est(k) = k·nz(k) + (64−k)·n (A-17, A-18)
  uint64_t best = ~0ull, nz = 0;
  for (uint32_t kk = 1; kk <= 64; ++kk) {
    nz += cnt[kk - 1];
    const uint64_t e = (uint64_t)kk * nz + (uint64_t)(64 - kk) * n;
    if (e < best) {
      best = e;
      k = kk;
    }
  }
  const uint32_t sh = 64 - k;
  const size_t L1 = cdiv(n, 8), L2 = cdiv(L1, 8), L3 = cdiv(L2, 8);
  uint8_t B1[kChunkBytes / 64 + 2] = {0}, B2[kChunkBytes / 512 + 2], B3[8];
  size_t nset = 0;
  uint64_t ptop = 0;
  for (size_t i = 0; i < n; ++i) {
    const uint64_t top = v[i] >> sh;
    if (rare ? top != ptop : top != 0) {
      B1[i >> 3] |= (uint8_t)(1u << (i & 7));
      ++nset;
    }
    ptop = top;
  }
  rep_bits(B1, L1, B2);
  rep_bits(B2, L2, B3);
  const size_t nr1 = popc_bits(B2, L1), nr2 = popc_bits(B3, L2);
  const size_t hib = cdiv(nset * k, 8), lob = cdiv(n * sh, 8);
  const size_t total = 3 + hib + lob + t + nr1 + nr2 + L3;
  if (total >= 3 + L) {  // bypass (A-23)
    out[0] = (uint8_t)L;
    out[1] = (uint8_t)(L >> 8);
    out[2] = 0;
    std::memcpy(out + 3, in, L);
    return 3 + L;
  }
  out[0] = (uint8_t)L;
  out[1] = (uint8_t)(L >> 8);
  out[2] = (uint8_t)k;
  {
    BitW hi(out + 3);
    for (size_t i = 0; i < n; ++i)
      if ((B1[i >> 3] >> (i & 7)) & 1) hi.put(v[i] >> sh, k);
    hi.finish();
  }
  if (sh) {
    const uint64_t lm = (1ull << sh) - 1;
    BitW lo(out + 3 + hib);
    for (size_t i = 0; i < n; ++i) lo.put(v[i] & lm, sh);
    lo.finish();
  }
  size_t o = 3 + hib + lob;
  std::memcpy(out + o, in + 8 * n, t);
  o += t;
  o += put_nr(B1, L1, B2, out + o);
  o += put_nr(B2, L2, B3, out + o);
  std::memcpy(out + o, B3, L3);
  return o + L3;
}
// in: len bytes (8 bytes of readable slack); out: capacity cap. Returns the
// decoded length or −1.
long adaptive_dec(const uint8_t* in, size_t len, uint8_t* out, size_t cap, bool rare) {
  if (len < 3) return -1;
  const size_t L = in[0] | ((size_t)in[1] << 8);
  const uint32_t k = in[2];
  if (L > cap) return -1;
  if (k == 0) {
    if (len != 3 + L) return -1;
    std::memcpy(out, in + 3, L);
    return (long)L;
  }
  if (k > 64) return -1;
  const uint32_t sh = 64 - k;
  const size_t n = L / 8, t = L % 8, L1 = cdiv(n, 8), L2 = cdiv(L1, 8), L3 = cdiv(L2, 8);
  uint8_t B1[kChunkBytes / 64 + 2], B2[kChunkBytes / 512 + 2];
  if (len < 3 + L3) return -1;
  const uint8_t* B3 = in + len - L3;
  const size_t c2 = popc_bits(B3, L2), s2 = len - L3 - c2;
  if (len - L3 < c2 || s2 < 3) return -1;
  get_nr(in + s2, B3, L2, B2);
  const size_t c1 = popc_bits(B2, L1);
  if (s2 < 3 + c1) return -1;
  const size_t s1 = s2 - c1;
  get_nr(in + s1, B2, L1, B1);
  const size_t nset = popc_bits(B1, n), hib = cdiv(nset * k, 8), lob = cdiv(n * sh, 8);
  if (3 + hib + lob + t != s1) return -1;
  BitR hi(in + 3), lo(in + 3 + hib);
  uint64_t ptop = 0;
  for (size_t i = 0; i < n; ++i) {
    const bool set = (B1[i >> 3] >> (i & 7)) & 1;
    const uint64_t top = set ? hi.get(k) : (rare ? ptop : 0ull);
    ptop = top;
    st64(out + 8 * i, sh ? ((top << sh) | lo.get(sh)) : top);
  }
  std::memcpy(out + 8 * n, in + 3 + hib + lob, t);
  return (long)L;
}

// ---- codec geometry ----
struct Geo {
  int algo;
  uint32_t wb;
  uint64_t n;   // words
  uint64_t C;   // chunks
  uint32_t cw;  // chunk words
  uint32_t words(uint64_t c) const {  // words of chunk c
    const uint64_t first = (algo == 3 ? c / 2 : c) * cw;
    return (uint32_t)std::min<uint64_t>(cw, n - first);
  }
  uint64_t raw_len(uint64_t c) const { return (uint64_t)words(c) * (algo == 3 ? 8 : wb); }
};
Geo geometry(int algo, uint64_t in_bytes) {
  Geo g;
  g.algo = algo;
  g.wb = word_bytes(algo);
  g.n = in_bytes / g.wb;
  g.cw = (uint32_t)(kChunkBytes / g.wb);
  g.C = algo == 3 ? 2 * cdiv(g.n, kTile) : cdiv(g.n, g.cw);
  return g;
}
size_t max_size(const Geo& g) {
  size_t s = r16(kHeader + 4 * g.C);
  for (uint64_t c = 0; c < g.C; ++c) s += r16(g.raw_len(c));
  return s;
}

// Encode chunk c's m words (already DIFFMS'd where the codec needs it) into
// buf; returns the encoded length (≥ raw length ⇒ the caller stores raw).
struct Scratch {
  std::unique_ptr<uint8_t[]> a{new uint8_t[kBuf]}, b{new uint8_t[kBuf]}, c{new uint8_t[kBuf]};
};
size_t encode_chunk(int algo, const uint8_t* words, uint32_t m, Scratch& S, const uint8_t** enc) {
  uint8_t* u = S.a.get();
  switch (algo) {
    case 0:
    case 2:
      if (algo == 0) diffms(reinterpret_cast<const uint32_t*>(words), reinterpret_cast<uint32_t*>(u), m);
      else diffms(reinterpret_cast<const uint64_t*>(words), reinterpret_cast<uint64_t*>(u), m);
      *enc = S.b.get();
      return algo == 0 ? mplg_enc(reinterpret_cast<const uint32_t*>(u), m, S.b.get())
                       : mplg_enc(reinterpret_cast<const uint64_t*>(u), m, S.b.get());
    case 1: {
      diffms(reinterpret_cast<const uint32_t*>(words), reinterpret_cast<uint32_t*>(u), m);
      bit_enc(reinterpret_cast<const uint32_t*>(u), m, reinterpret_cast<uint32_t*>(S.c.get()));
      *enc = S.b.get();
      return rze_enc(S.c.get(), 4 * (size_t)m, S.b.get());
    }
    default: {  // DPratio chunk (V or Dist words)
      diffms(reinterpret_cast<const uint64_t*>(words), reinterpret_cast<uint64_t*>(u), m);
      const size_t l1 = adaptive_enc(u, 8 * (size_t)m, S.c.get(), false);
      *enc = S.b.get();
      return adaptive_enc(S.c.get(), l1, S.b.get(), true);
    }
  }
}
// Decode a non-raw payload (copied to pay with slack) into out (raw_len bytes).
bool decode_chunk(int algo, const uint8_t* pay, size_t len, uint32_t m, uint8_t* out, Scratch& S) {
  switch (algo) {
    case 0: return mplg_dec(pay, len, reinterpret_cast<uint32_t*>(out), m);
    case 2: return mplg_dec(pay, len, reinterpret_cast<uint64_t*>(out), m);
    case 1: {
      uint8_t* T = S.c.get();
      if (!rze_dec(pay, len, T, 4 * (size_t)m)) return false;
      bit_dec(reinterpret_cast<const uint32_t*>(T), m, reinterpret_cast<uint32_t*>(out));
      undiffms(reinterpret_cast<uint32_t*>(out), m);
      return true;
    }
    default: {
      uint8_t* r = S.c.get();
      const long l1 = adaptive_dec(pay, len, r, kChunkBytes + 3, true);
      if (l1 < 0) return false;
      std::memset(r + l1, 0, 16);  // slack for the bit readers
      if (adaptive_dec(r, (size_t)l1, out, 8 * (size_t)m, false) != (long)(8 * m)) return false;
      undiffms(reinterpret_cast<uint64_t*>(out), m);
      return true;
    }
  }
}

template <class F> void parallel(int nt, F&& f) {
  std::vector<std::thread> th;
  for (int t = 1; t < nt; ++t) th.emplace_back(f, t);
  f(0);
  for (auto& x : th) x.join();
}
int threads_of(int n_threads) {
  if (n_threads > 0) return n_threads;
  const unsigned h = std::thread::hardware_concurrency();
  return h ? (int)h : 1;
}

// ---- FCM (FORMAT.md §6.1): V and Dist of the whole array ----
constexpr uint64_t K1 = 0x9E3779B97F4A7C15ull, K2 = 0xC2B2AE3D27D4EB4Full, K3 = 0x165667B19E3779F9ull;
// A record is h (20 bits) | fp (12 bits, a fingerprint of x[i] that only
// filters candidates: x itself is compared on a fingerprint hit) | i (32 bits).
inline uint64_t fcm_rec(uint64_t h, uint64_t xi, uint64_t i) {
  const uint32_t f = (uint32_t)(xi ^ (xi >> 32));
  return (h << 44) | ((uint64_t)((f ^ (f >> 12) ^ (f >> 24)) & 0xFFFu) << 32) | i;
}
void fcm_encode(const uint64_t* x, uint64_t n, uint64_t* V, uint64_t* Dist, int nt) {
  std::vector<uint64_t> a(n), b(n);
  const uint64_t per = cdiv(n, (uint64_t)nt);
  parallel(nt, [&](int t) {
    const uint64_t i0 = std::min(n, t * per), i1 = std::min(n, i0 + per);
    for (uint64_t i = i0; i < i1; ++i) {
      const uint64_t p1 = i >= 1 ? x[i - 1] : 0, p2 = i >= 2 ? x[i - 2] : 0, p3 = i >= 3 ? x[i - 3] : 0;
      const uint64_t h = ((p1 * K1) ^ (p2 * K2) ^ (p3 * K3)) >> 44;
      a[i] = fcm_rec(h, x[i], i);
      Dist[i] = 0;
    }
  });
  // stable LSD radix sort on the two 10-bit digits of h: per-thread counts,
  // (digit, thread)-major prefix, scatter
  std::vector<uint64_t> cnt((size_t)nt * 1024);
  for (int pass = 0; pass < 2; ++pass) {
    const int shift = 44 + 10 * pass;
    const uint64_t* src = pass ? b.data() : a.data();
    uint64_t* dst = pass ? a.data() : b.data();
    parallel(nt, [&](int t) {
      uint64_t* c = &cnt[(size_t)t * 1024];
      std::fill(c, c + 1024, 0);
      const uint64_t i0 = std::min(n, t * per), i1 = std::min(n, i0 + per);
      for (uint64_t i = i0; i < i1; ++i) ++c[(src[i] >> shift) & 1023];
    });
    uint64_t run = 0;
    for (int d = 0; d < 1024; ++d)
      for (int t = 0; t < nt; ++t) {
        const uint64_t v = cnt[(size_t)t * 1024 + d];
        cnt[(size_t)t * 1024 + d] = run;
        run += v;
      }
    parallel(nt, [&](int t) {
      uint64_t* c = &cnt[(size_t)t * 1024];
      const uint64_t i0 = std::min(n, t * per), i1 = std::min(n, i0 + per);
      for (uint64_t i = i0; i < i1; ++i) dst[c[(src[i] >> shift) & 1023]++] = src[i];
    });
  }
  // a = records sorted by (h, i); the nearest of the ≤ 4 preceding pairs with
  // the same hash and an equal word (A-14, A-15); only matches are written
  parallel(nt, [&](int t) {
    const uint64_t k0 = std::min(n, t * per), k1 = std::min(n, k0 + per);
    for (uint64_t k = k0; k < k1; ++k) {
      const uint64_t rk = a[k], i = rk & 0xFFFFFFFFull;
      for (uint64_t back = 1; back <= 4 && back <= k; ++back) {
        const uint64_t rb = a[k - back];
        if ((rb >> 44) != (rk >> 44)) break;  // left the hash's run
        const uint64_t j = rb & 0xFFFFFFFFull;
        if ((rb >> 32) == (rk >> 32) && x[j] == x[i]) {
          Dist[i] = i - j;
          break;
        }
      }
    }
  });
  parallel(nt, [&](int t) {
    const uint64_t i0 = std::min(n, t * per), i1 = std::min(n, i0 + per);
    for (uint64_t i = i0; i < i1; ++i) V[i] = Dist[i] ? 0 : x[i];
  });
}

// ---- stream ----
void write_header(uint8_t* out, int algo, uint32_t wb, uint64_t n_bytes, uint64_t C, uint64_t payload) {
  std::memset(out, 0, kHeader);
  st32(out, kMagic);
  out[4] = 1;
  out[5] = (uint8_t)algo;
  out[6] = (uint8_t)wb;
  st64(out + 8, n_bytes);
  st64(out + 16, C);
  st64(out + 24, payload);
}

int compress(int algo, int dtype, const uint8_t* in, size_t in_bytes, uint8_t* out, size_t cap, size_t* out_bytes,
             int n_threads) {
  const uint32_t wb = word_bytes(algo);
  if (!wb) return kInvalid;
  if (!dtype_ok(algo, dtype)) return kDtype;
  if (in_bytes % wb) return kInvalid;
  const Geo g = geometry(algo, in_bytes);
  if (algo == 3 && g.n > 0xFFFFFFFFull) return kInvalid;  // 32-bit FCM indices
  if (cap < max_size(g)) return kSmall;
  const int nt = (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)threads_of(n_threads), std::max<uint64_t>(g.C, 1)));
  const size_t base = r16(kHeader + 4 * g.C);
  std::memset(out + kHeader + 4 * g.C, 0, base - kHeader - 4 * g.C);
  // DPratio: FCM over the whole array first (L104)
  std::vector<uint64_t> V, Dist;
  if (algo == 3 && g.n) {
    V.resize(g.n);
    Dist.resize(g.n);
    fcm_encode(reinterpret_cast<const uint64_t*>(in), g.n, V.data(), Dist.data(),
               (int)std::max(1, std::min<int>(threads_of(n_threads), (int)std::min<uint64_t>(g.n / 65536 + 1, 1024))));
  }
  std::atomic<uint64_t> next{0};
  std::unique_ptr<std::atomic<uint64_t>[]> end(new (std::nothrow) std::atomic<uint64_t>[std::max<uint64_t>(g.C, 1)]);
  if (!end) return kOom;
  for (uint64_t c = 0; c < g.C; ++c) end[c].store(~0ull, std::memory_order_relaxed);
  uint8_t* table = out + kHeader;
  uint8_t* pay = out + base;
  parallel(nt, [&](int) {
    Scratch S;
    std::vector<uint8_t> words(kChunkBytes);
    for (;;) {
      const uint64_t c = next.fetch_add(1, std::memory_order_relaxed);  // dynamic worklist (L104)
      if (c >= g.C) return;
      const uint32_t m = g.words(c);
      const uint8_t* src;
      if (algo == 3) {
        const uint64_t t0 = (c / 2) * kTile;
        src = reinterpret_cast<const uint8_t*>((c & 1 ? Dist.data() : V.data()) + t0);
      } else {
        src = in + c * kChunkBytes;
      }
      const uint8_t* enc = nullptr;
      size_t len = encode_chunk(algo, src, m, S, &enc);
      const size_t raw = g.raw_len(c);
      const bool is_raw = len >= raw;  // L104, ties → raw
      if (is_raw) {
        enc = src;
        len = raw;
      }
      // write position from the previous chunk (L120), then ours for the next
      uint64_t start = 0;
      if (c) {
        while ((start = end[c - 1].load(std::memory_order_acquire)) == ~0ull) std::this_thread::yield();
      }
      end[c].store(start + r16(len), std::memory_order_release);
      std::memcpy(pay + start, enc, len);
      std::memset(pay + start + len, 0, r16(len) - len);
      st32(table + 4 * c, (uint32_t)len | (is_raw ? kRawFlag : 0u));
    }
  });
  const uint64_t payload = g.C ? end[g.C - 1].load() : 0;
  write_header(out, algo, wb, in_bytes, g.C, payload);
  if (out_bytes) *out_bytes = base + payload;
  return kOk;
}

int decompress(int algo, int dtype, const uint8_t* in, size_t in_bytes, uint8_t* out, size_t cap, size_t* out_bytes,
               int n_threads) {
  const uint32_t wb = word_bytes(algo);
  if (!wb) return kInvalid;
  if (!dtype_ok(algo, dtype)) return kDtype;
  if (in_bytes < kHeader) return kCorrupt;
  if (ld32(in) != kMagic || in[4] != 1 || in[7] != 0 || in[5] > 3) return kCorrupt;
  if (in[5] != algo) return kDtype;
  if (in[6] != wb) return kCorrupt;
  const uint64_t n_bytes = ld64(in + 8), C = ld64(in + 16), payload = ld64(in + 24);
  if (n_bytes % wb) return kCorrupt;
  const Geo g = geometry(algo, n_bytes);
  if (C != g.C || C > (in_bytes - kHeader) / 4) return kCorrupt;
  const uint64_t base = r16(kHeader + 4 * C);
  if (base > in_bytes || payload > in_bytes - base) return kCorrupt;
  if (cap < n_bytes) return kSmall;
  // read offsets: prefix sum of the padded sizes (L120)
  std::vector<uint64_t> off(C + 1);
  for (uint64_t c = 0; c < C; ++c) {
    const uint32_t e = ld32(in + kHeader + 4 * c), len = e & ~kRawFlag;
    const uint64_t raw = g.raw_len(c);
    if ((e & kRawFlag) ? len != raw : len >= raw) return kCorrupt;
    off[c + 1] = off[c] + r16(len);
  }
  if (off[C] != payload) return kCorrupt;
  const int nt = (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)threads_of(n_threads), std::max<uint64_t>(C, 1)));
  std::vector<uint64_t> Dist(algo == 3 ? g.n : 0);
  std::atomic<uint64_t> next{0};
  std::atomic<int> bad{0};
  const uint8_t* pay = in + base;
  parallel(nt, [&](int) {
    Scratch S;
    std::vector<uint8_t> buf(kBuf);
    for (;;) {
      const uint64_t c = next.fetch_add(1, std::memory_order_relaxed);
      if (c >= C || bad.load(std::memory_order_relaxed)) return;
      const uint32_t e = ld32(in + kHeader + 4 * c), len = e & ~kRawFlag;
      const uint32_t m = g.words(c);
      uint8_t* dst;
      if (algo == 3) {
        const uint64_t t0 = (c / 2) * kTile;
        dst = c & 1 ? reinterpret_cast<uint8_t*>(Dist.data() + t0) : out + 8 * t0;
      } else {
        dst = out + c * kChunkBytes;
      }
      if (e & kRawFlag) {
        std::memcpy(dst, pay + off[c], len);
        continue;
      }
      std::memcpy(buf.data(), pay + off[c], len);  // with zeroed slack for the bit readers
      std::memset(buf.data() + len, 0, 16);
      if (!decode_chunk(algo, buf.data(), len, m, dst, S)) bad.store(1);
    }
  });
  if (bad.load()) return kCorrupt;
  if (algo == 3 && g.n) {
    // FCM decode (L197): x[i] = Dist[i] ? x[i − Dist[i]] : V[i], V already in
    // out. Tiles go to threads in index order; a tile that references an
    // earlier tile waits for that tile's flag (claimed earlier ⇒ no deadlock).
    uint64_t* x = reinterpret_cast<uint64_t*>(out);
    const uint64_t T = cdiv(g.n, kTile);
    std::unique_ptr<std::atomic<uint8_t>[]> done(new std::atomic<uint8_t>[T]);
    for (uint64_t t = 0; t < T; ++t) done[t].store(0, std::memory_order_relaxed);
    std::atomic<uint64_t> nt2{0};
    parallel(nt, [&](int) {
      for (;;) {
        const uint64_t t = nt2.fetch_add(1, std::memory_order_relaxed);
        if (t >= T) return;
        const uint64_t i0 = t * kTile, i1 = std::min<uint64_t>(g.n, i0 + kTile);
        for (uint64_t i = i0; i < i1; ++i) {
          const uint64_t d = Dist[i];
          if (!d) continue;
          if (d > i || x[i] != 0) {
            bad.store(1);
            break;
          }
          const uint64_t j = i - d;
          if (j < i0)
            while (!done[j / kTile].load(std::memory_order_acquire)) std::this_thread::yield();
          x[i] = x[j];
        }
        done[t].store(1, std::memory_order_release);
      }
    });
    if (bad.load()) return kCorrupt;
  }
  if (out_bytes) *out_bytes = n_bytes;
  return kOk;
}

}  // namespace

extern "C" {

size_t lcf_cpu_max_compressed_size(int algo, int dtype, size_t in_bytes) {
  (void)dtype;
  if (!word_bytes(algo)) return 0;
  return max_size(geometry(algo, in_bytes - in_bytes % word_bytes(algo)));
}

int lcf_cpu_compress(int algo, int dtype, const void* in, size_t in_bytes, void* out, size_t out_capacity,
                     size_t* out_bytes, int n_threads) {
  if ((!in && in_bytes) || !out) return kInvalid;
  try {
    return compress(algo, dtype, static_cast<const uint8_t*>(in), in_bytes, static_cast<uint8_t*>(out),
                    out_capacity, out_bytes, n_threads);
  } catch (const std::bad_alloc&) {
    return kOom;
  }
}

int lcf_cpu_decompress(int algo, int dtype, const void* in, size_t in_bytes, void* out, size_t out_capacity,
                       size_t* out_bytes, int n_threads) {
  if (!in || (!out && out_capacity)) return kInvalid;
  try {
    return decompress(algo, dtype, static_cast<const uint8_t*>(in), in_bytes, static_cast<uint8_t*>(out),
                      out_capacity, out_bytes, n_threads);
  } catch (const std::bad_alloc&) {
    return kOom;
  }
}

}  // extern "C"
