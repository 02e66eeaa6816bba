// lcf_oracle.cpp — plain CPU oracle (TEST INFRASTRUCTURE ONLY; see lcf_oracle.h).
//
// Written from PAPER.md (cited as L<line>) and FORMAT.md, step by step, in the
// paper's order. Deliberately naive: bit streams are written one bit at a time,
// bitmaps one bit at a time, FCM uses std::sort. Nothing here is shared with
// the CUDA path.
#include "lcf_oracle.h"

#include <algorithm>
#include <cstring>
#include <type_traits>
#include <utility>
#include <vector>

namespace {

using Bytes = std::vector<uint8_t>;

enum { OK = 0, E_ARG = 1, E_DTYPE = 2, E_SMALL = 3, E_CORRUPT = 4 };
enum { SPSPEED = 0, SPRATIO = 1, DPSPEED = 2, DPRATIO = 3 };

size_t round_up(size_t v, size_t a) { return (v + a - 1) / a * a; }
size_t ceil_div(size_t v, size_t a) { return (v + a - 1) / a; }

// ---------------------------------------------------------------------------
// Bit streams, LSB-first (FORMAT.md preamble). One bit at a time.
// ---------------------------------------------------------------------------
void put_bits(Bytes& s, uint64_t& pos, uint64_t v, unsigned w) {
  for (unsigned j = 0; j < w; ++j) {
    if (pos / 8 >= s.size()) s.push_back(0);
    if ((v >> j) & 1u) s[pos / 8] |= (uint8_t)(1u << (pos % 8));
    ++pos;
  }
}
uint64_t get_bits(const uint8_t* s, uint64_t& pos, unsigned w) {
  uint64_t v = 0;
  for (unsigned j = 0; j < w; ++j) {
    if ((s[pos / 8] >> (pos % 8)) & 1u) v |= (uint64_t)1 << j;
    ++pos;
  }
  return v;
}

template <class U> unsigned bitlen(U v) {  // W − clz_W(v); bitlen(0) = 0
  unsigned b = 0;
  while (v) { ++b; v >>= 1; }
  return b;
}
template <class U> unsigned clz(U v) { return (unsigned)(sizeof(U) * 8) - bitlen(v); }

template <class U> U load_le(const uint8_t* p) {
  U v = 0;
  for (size_t b = 0; b < sizeof(U); ++b) v |= (U)p[b] << (8 * b);
  return v;
}
template <class U> void store_le(uint8_t* p, U v) {
  for (size_t b = 0; b < sizeof(U); ++b) p[b] = (uint8_t)(v >> (8 * b));
}

// ---------------------------------------------------------------------------
// DIFFMS (L110–112): difference mod 2^W to the preceding value (first value
// against 0, "as if 0 was its preceding value"), then two's complement →
// magnitude-sign "(data << 1) ^ (data >> 31)" with an arithmetic right shift.
// ---------------------------------------------------------------------------
template <class U> U tcms(U d) {  // L112
  using S = std::make_signed_t<U>;
  const unsigned W = sizeof(U) * 8;
  return (U)(d << 1) ^ (U)((S)d >> (W - 1));
}
template <class U> U tcms_inv(U u) { return (U)(u >> 1) ^ (U)(0 - (u & 1u)); }

template <class U> void diffms_enc(const U* x, size_t n, U* u) {
  U prev = 0;
  for (size_t i = 0; i < n; ++i) {
    u[i] = tcms<U>((U)(x[i] - prev));
    prev = x[i];
  }
}
template <class U> void diffms_dec(const U* u, size_t n, U* x) {
  U prev = 0;
  for (size_t i = 0; i < n; ++i) {
    x[i] = (U)(prev + tcms_inv<U>(u[i]));
    prev = x[i];
  }
}

// ---------------------------------------------------------------------------
// MPLG, enhanced (L114–118, Fig. 3): per 512-byte subchunk find the
// maximum, eliminate its leading zero bits from every value; if the maximum
// has no leading zero, first apply TCMS once more to the subchunk (A-7).
// ---------------------------------------------------------------------------
template <class U> Bytes mplg_enc(const U* u, size_t n) {
  const unsigned W = sizeof(U) * 8;
  const size_t SW = 512 / sizeof(U);
  const size_t S = ceil_div(n, SW);
  Bytes out(round_up(S, 8), 0);  // header: one byte per subchunk (A-8)
  for (size_t s = 0; s < S; ++s) {
    const size_t ms = std::min(SW, n - s * SW);
    std::vector<U> v(u + s * SW, u + s * SW + ms);
    U M = *std::max_element(v.begin(), v.end());
    unsigned flag = 0;
    if (clz<U>(M) == 0) {  // "If the maximum has no leading zeros" (L114)
      flag = 1;
      for (U& e : v) e = tcms<U>(e);
      M = *std::max_element(v.begin(), v.end());
    }
    const unsigned w = W - clz<U>(M);  // keep w low bits (L116)
    out[s] = (uint8_t)(w | (flag << 7));
    Bytes bs;
    uint64_t pos = 0;
    for (size_t j = 0; j < ms; ++j) put_bits(bs, pos, (uint64_t)v[j], w);
    bs.resize(ceil_div(ms * w, 8), 0);
    out.insert(out.end(), bs.begin(), bs.end());
  }
  return out;
}
template <class U> int mplg_dec(const uint8_t* in, size_t len, size_t n, U* u) {
  const unsigned W = sizeof(U) * 8;
  const size_t SW = 512 / sizeof(U);
  const size_t S = ceil_div(n, SW);
  size_t off = round_up(S, 8);
  if (off > len) return E_CORRUPT;
  for (size_t s = 0; s < S; ++s) {
    const size_t ms = std::min(SW, n - s * SW);
    const unsigned w = in[s] & 0x7Fu, flag = in[s] >> 7;
    if (w > W) return E_CORRUPT;
    const size_t nb = ceil_div(ms * w, 8);
    if (off + nb > len) return E_CORRUPT;
    uint64_t pos = 0;
    for (size_t j = 0; j < ms; ++j) {
      U v = (U)get_bits(in + off, pos, w);
      u[s * SW + j] = flag ? tcms_inv<U>(v) : v;
    }
    off += nb;
  }
  return off == len ? OK : E_CORRUPT;
}

// ---------------------------------------------------------------------------
// BIT (L140–142, Fig. 4): bit transposition. Plane-major over the
// chunk, most-significant plane first, value i of a 32-value group ↦ bit i
// (A-9). Leftover m mod 32 words are copied.
// ---------------------------------------------------------------------------
void bit32_enc(const uint32_t* u, size_t m, uint32_t* T) {
  const size_t G = m / 32;
  for (size_t g = 0; g < G; ++g)
    for (size_t p = 0; p < 32; ++p) {
      uint32_t word = 0;
      for (size_t i = 0; i < 32; ++i) word |= ((u[32 * g + i] >> (31 - p)) & 1u) << i;
      T[p * G + g] = word;
    }
  for (size_t i = 32 * G; i < m; ++i) T[i] = u[i];
}
void bit32_dec(const uint32_t* T, size_t m, uint32_t* u) {
  const size_t G = m / 32;
  for (size_t g = 0; g < G; ++g)
    for (size_t i = 0; i < 32; ++i) {
      uint32_t word = 0;
      for (size_t p = 0; p < 32; ++p) word |= ((T[p * G + g] >> i) & 1u) << (31 - p);
      u[32 * g + i] = word;
    }
  for (size_t i = 32 * G; i < m; ++i) u[i] = T[i];
}

// ---------------------------------------------------------------------------
// Repetition elimination of a bitmap (L146): next-level bitmap bit j is set iff
// byte j differs from byte j−1 (byte −1 = 0); the differing bytes are kept.
// ---------------------------------------------------------------------------
void repeat_elim(const Bytes& B, Bytes& next, Bytes& kept) {
  next.assign(ceil_div(B.size(), 8), 0);
  kept.clear();
  for (size_t j = 0; j < B.size(); ++j) {
    const uint8_t prev = j ? B[j - 1] : 0;
    if (B[j] != prev) {
      next[j / 8] |= (uint8_t)(1u << (j % 8));
      kept.push_back(B[j]);
    }
  }
}
size_t popcount_bits(const uint8_t* bm, size_t nbits) {
  size_t c = 0;
  for (size_t j = 0; j < nbits; ++j) c += (bm[j / 8] >> (j % 8)) & 1u;
  return c;
}
// Inverse: rebuild Lb bytes from the next-level bitmap and the kept bytes that
// end at in[end]. Returns the start of the kept bytes, or SIZE_MAX if corrupt.
size_t repeat_restore(const uint8_t* in, size_t end, const Bytes& next, size_t Lb, Bytes& B) {
  const size_t cnt = popcount_bits(next.data(), Lb);
  if (cnt > end) return SIZE_MAX;
  const size_t start = end - cnt;
  B.assign(Lb, 0);
  size_t r = 0;
  for (size_t j = 0; j < Lb; ++j) {
    if ((next[j / 8] >> (j % 8)) & 1u) B[j] = in[start + r++];
    else B[j] = j ? B[j - 1] : 0;
  }
  return start;
}

// ---------------------------------------------------------------------------
// RZE (L144–148, L158): bitmap of non-zero bytes + the non-zero bytes; the
// bitmap is compressed three times by repetition elimination (16384 → 2048 →
// 256 → 32 bits); output = non-zero bytes followed by the compressed bitmap.
// ---------------------------------------------------------------------------
Bytes rze_enc(const uint8_t* D, size_t L) {
  Bytes B1(ceil_div(L, 8), 0), nz;
  for (size_t i = 0; i < L; ++i)
    if (D[i] != 0) {
      B1[i / 8] |= (uint8_t)(1u << (i % 8));
      nz.push_back(D[i]);
    }
  Bytes B2, B3, B4, nr1, nr2, nr3;
  repeat_elim(B1, B2, nr1);
  repeat_elim(B2, B3, nr2);
  repeat_elim(B3, B4, nr3);
  Bytes out = nz;
  out.insert(out.end(), nr1.begin(), nr1.end());
  out.insert(out.end(), nr2.begin(), nr2.end());
  out.insert(out.end(), nr3.begin(), nr3.end());
  out.insert(out.end(), B4.begin(), B4.end());
  return out;
}
int rze_dec(const uint8_t* in, size_t len, size_t L, uint8_t* D) {
  const size_t L1 = ceil_div(L, 8), L2 = ceil_div(L1, 8), L3 = ceil_div(L2, 8),
               L4 = ceil_div(L3, 8);
  if (L4 > len) return E_CORRUPT;
  Bytes B4(in + len - L4, in + len), B3, B2, B1;
  size_t end = len - L4;
  end = repeat_restore(in, end, B4, L3, B3);
  if (end == SIZE_MAX) return E_CORRUPT;
  end = repeat_restore(in, end, B3, L2, B2);
  if (end == SIZE_MAX) return E_CORRUPT;
  end = repeat_restore(in, end, B2, L1, B1);
  if (end == SIZE_MAX) return E_CORRUPT;
  if (popcount_bits(B1.data(), L) != end) return E_CORRUPT;  // nz(D) = in[0, end)
  size_t r = 0;
  for (size_t i = 0; i < L; ++i) D[i] = ((B1[i / 8] >> (i % 8)) & 1u) ? in[r++] : 0;
  return OK;
}

// ---------------------------------------------------------------------------
// FCM (L170–185, Fig. 6): pairs (hash of the three prior values, index),
// sorted; a pair matches one of the preceding four sorted pairs with the same
// hash and the same value (nearest first, A-14) → V = 0, Dist = distance;
// otherwise V = value, Dist = 0.
// ---------------------------------------------------------------------------
const uint64_t FCM_K1 = 0x9E3779B97F4A7C15ull, FCM_K2 = 0xC2B2AE3D27D4EB4Full,
               FCM_K3 = 0x165667B19E3779F9ull;  // A-13
void fcm_hash(const uint64_t* x, size_t n, uint32_t* h) {
  for (size_t i = 0; i < n; ++i) {
    const uint64_t a = i >= 1 ? x[i - 1] : 0, b = i >= 2 ? x[i - 2] : 0, c = i >= 3 ? x[i - 3] : 0;
    h[i] = (uint32_t)(((a * FCM_K1) ^ (b * FCM_K2) ^ (c * FCM_K3)) >> 44);
  }
}
void fcm_match(const uint64_t* x, const uint32_t* h, size_t n, uint64_t* V, uint64_t* Dist) {
  std::vector<std::pair<uint32_t, uint64_t>> P(n);
  for (size_t i = 0; i < n; ++i) P[i] = {h[i], (uint64_t)i};
  std::sort(P.begin(), P.end());
  for (size_t k = 0; k < n; ++k) {
    const uint64_t i = P[k].second;
    V[i] = x[i];
    Dist[i] = 0;
    for (size_t d = 1; d <= 4 && d <= k; ++d) {
      if (P[k - d].first != P[k].first) continue;
      const uint64_t j = P[k - d].second;
      if (x[j] == x[i]) {
        V[i] = 0;
        Dist[i] = i - j;
        break;
      }
    }
  }
}
int fcm_dec(const uint64_t* V, const uint64_t* Dist, size_t n, uint64_t* x) {
  for (size_t i = 0; i < n; ++i) {
    if (Dist[i] == 0) x[i] = V[i];
    else {
      if (Dist[i] > i || V[i] != 0) return E_CORRUPT;
      x[i] = x[i - Dist[i]];
    }
  }
  return OK;
}

// ---------------------------------------------------------------------------
// RAZE (L189, Fig. 7) and RARE (L195): split each 64-bit word into its top k
// and low 64−k bits with k chosen per chunk from a histogram of leading-zero
// counts and its prefix sum; zero-eliminate (RAZE) or repetition-eliminate
// (RARE) the top parts with a bitmap compressed twice more by repetition
// elimination; keep the low parts.
// ---------------------------------------------------------------------------
Bytes adaptive_enc(const uint8_t* in, size_t L, bool rare) {
  const size_t n = L / 8, t = L % 8;
  std::vector<uint64_t> v(n);
  for (size_t i = 0; i < n; ++i) v[i] = load_le<uint64_t>(in + 8 * i);
  auto ref = [&](size_t i) -> uint64_t { return (rare && i > 0) ? v[i - 1] : 0; };
  // histogram of leading-zero counts (65 bins, A-17), prefix sum, size per k
  std::vector<uint64_t> cnt(65, 0);
  for (size_t i = 0; i < n; ++i) cnt[clz<uint64_t>(v[i] ^ ref(i))]++;
  unsigned k = 1;
  uint64_t best = UINT64_MAX;
  for (unsigned kk = 1; kk <= 64; ++kk) {
    uint64_t nzk = 0;
    for (unsigned z = 0; z < kk; ++z) nzk += cnt[z];
    const uint64_t est = (uint64_t)kk * nzk + (uint64_t)(64 - kk) * n;  // A-18
    if (est < best) { best = est; k = kk; }
  }
  auto top = [&](uint64_t w) -> uint64_t { return k == 64 ? w : w >> (64 - k); };
  auto low = [&](uint64_t w) -> uint64_t { return k == 64 ? 0 : w & ((1ull << (64 - k)) - 1); };
  Bytes B1(ceil_div(n, 8), 0), HI, LO;
  uint64_t phi = 0, plo = 0;
  for (size_t i = 0; i < n; ++i) {
    const uint64_t tp = top(v[i]);
    const uint64_t tref = rare ? (i ? top(v[i - 1]) : 0) : 0;
    if (tp != tref) {
      B1[i / 8] |= (uint8_t)(1u << (i % 8));
      put_bits(HI, phi, tp, k);
    }
  }
  HI.resize(ceil_div(phi, 8), 0);
  for (size_t i = 0; i < n; ++i) put_bits(LO, plo, low(v[i]), 64 - k);
  LO.resize(ceil_div(plo, 8), 0);
  Bytes B2, B3, nr1, nr2;
  repeat_elim(B1, B2, nr1);
  repeat_elim(B2, B3, nr2);
  Bytes out = {(uint8_t)(L & 0xFF), (uint8_t)(L >> 8), (uint8_t)k};
  out.insert(out.end(), HI.begin(), HI.end());
  out.insert(out.end(), LO.begin(), LO.end());
  out.insert(out.end(), in + 8 * n, in + 8 * n + t);
  out.insert(out.end(), nr1.begin(), nr1.end());
  out.insert(out.end(), nr2.begin(), nr2.end());
  out.insert(out.end(), B3.begin(), B3.end());
  if (out.size() >= 3 + L) {  // per-stage bypass (A-23)
    out = {(uint8_t)(L & 0xFF), (uint8_t)(L >> 8), 0};
    out.insert(out.end(), in, in + L);
  }
  return out;
}
int adaptive_dec(const uint8_t* in, size_t len, bool rare, Bytes& out) {
  if (len < 3) return E_CORRUPT;
  const size_t L = (size_t)in[0] | ((size_t)in[1] << 8);
  const unsigned k = in[2];
  if (k == 0) {
    if (len != 3 + L) return E_CORRUPT;
    out.assign(in + 3, in + 3 + L);
    return OK;
  }
  if (k > 64) return E_CORRUPT;
  const size_t n = L / 8, t = L % 8;
  const size_t L1 = ceil_div(n, 8), L2 = ceil_div(L1, 8), L3 = ceil_div(L2, 8);
  if (3 + L3 > len) return E_CORRUPT;
  Bytes B3(in + len - L3, in + len), B2, B1;
  size_t end = len - L3;
  end = repeat_restore(in, end, B3, L2, B2);
  if (end == SIZE_MAX) return E_CORRUPT;
  end = repeat_restore(in, end, B2, L1, B1);
  if (end == SIZE_MAX) return E_CORRUPT;
  const size_t nset = popcount_bits(B1.data(), n);
  const size_t hib = ceil_div(nset * k, 8), lob = ceil_div(n * (64 - k), 8);
  if (3 + hib + lob + t != end) return E_CORRUPT;
  out.assign(L, 0);
  uint64_t phi = 0, plo = 0, prev_top = 0;
  for (size_t i = 0; i < n; ++i) {
    uint64_t tp;
    if ((B1[i / 8] >> (i % 8)) & 1u) tp = get_bits(in + 3, phi, k);
    else tp = rare ? prev_top : 0;
    prev_top = tp;
    const uint64_t lw = get_bits(in + 3 + hib, plo, 64 - k);
    const uint64_t w = k == 64 ? tp : (tp << (64 - k)) | lw;
    store_le<uint64_t>(out.data() + 8 * i, w);
  }
  std::memcpy(out.data() + 8 * n, in + 3 + hib + lob, t);
  return OK;
}

// ---------------------------------------------------------------------------
// Codec pipelines (L350): SPspeed = MPLG32∘DIFFMS32, DPspeed = MPLG64∘DIFFMS64,
// SPratio = RZE∘BIT32∘DIFFMS32, DPratio = per chunk RARE∘RAZE∘DIFFMS64 over
// FCM's V and Dist arrays. Decompression inverts the stages in reverse order
// (L94).
// ---------------------------------------------------------------------------
size_t word_bytes_of(int algo) { return (algo == SPSPEED || algo == SPRATIO) ? 4 : 8; }

Bytes encode_chunk(int algo, const uint8_t* raw, size_t m) {
  if (algo == SPSPEED || algo == SPRATIO) {
    std::vector<uint32_t> x(m), u(m);
    for (size_t i = 0; i < m; ++i) x[i] = load_le<uint32_t>(raw + 4 * i);
    diffms_enc<uint32_t>(x.data(), m, u.data());
    if (algo == SPSPEED) return mplg_enc<uint32_t>(u.data(), m);
    std::vector<uint32_t> T(m);
    bit32_enc(u.data(), m, T.data());
    Bytes D(4 * m);
    for (size_t i = 0; i < m; ++i) store_le<uint32_t>(D.data() + 4 * i, T[i]);
    return rze_enc(D.data(), D.size());
  }
  std::vector<uint64_t> x(m), u(m);
  for (size_t i = 0; i < m; ++i) x[i] = load_le<uint64_t>(raw + 8 * i);
  diffms_enc<uint64_t>(x.data(), m, u.data());
  if (algo == DPSPEED) return mplg_enc<uint64_t>(u.data(), m);
  Bytes D(8 * m);
  for (size_t i = 0; i < m; ++i) store_le<uint64_t>(D.data() + 8 * i, u[i]);
  Bytes r1 = adaptive_enc(D.data(), D.size(), false);  // RAZE
  return adaptive_enc(r1.data(), r1.size(), true);     // RARE
}

int decode_chunk(int algo, const uint8_t* in, size_t len, size_t m, uint8_t* raw) {
  if (algo == SPSPEED || algo == SPRATIO) {
    std::vector<uint32_t> u(m), x(m);
    if (algo == SPSPEED) {
      if (int st = mplg_dec<uint32_t>(in, len, m, u.data())) return st;
    } else {
      Bytes D(4 * m);
      if (int st = rze_dec(in, len, 4 * m, D.data())) return st;
      std::vector<uint32_t> T(m);
      for (size_t i = 0; i < m; ++i) T[i] = load_le<uint32_t>(D.data() + 4 * i);
      bit32_dec(T.data(), m, u.data());
    }
    diffms_dec<uint32_t>(u.data(), m, x.data());
    for (size_t i = 0; i < m; ++i) store_le<uint32_t>(raw + 4 * i, x[i]);
    return OK;
  }
  std::vector<uint64_t> u(m), x(m);
  if (algo == DPSPEED) {
    if (int st = mplg_dec<uint64_t>(in, len, m, u.data())) return st;
  } else {
    Bytes r1, D;
    if (int st = adaptive_dec(in, len, true, r1)) return st;  // RARE⁻¹
    if (int st = adaptive_dec(r1.data(), r1.size(), false, D)) return st;  // RAZE⁻¹
    if (D.size() != 8 * m) return E_CORRUPT;
    for (size_t i = 0; i < m; ++i) u[i] = load_le<uint64_t>(D.data() + 8 * i);
  }
  diffms_dec<uint64_t>(u.data(), m, x.data());
  for (size_t i = 0; i < m; ++i) store_le<uint64_t>(raw + 8 * i, x[i]);
  return OK;
}

// The chunk list of FORMAT.md §2 as (raw bytes, word count) pairs.
struct ChunkList {
  std::vector<Bytes> raw;
  std::vector<size_t> words;
};
ChunkList make_chunks(int algo, const uint8_t* in, size_t in_bytes) {
  ChunkList cl;
  const size_t wb = word_bytes_of(algo), n = in_bytes / wb, CW = 16384 / wb;
  if (algo != DPRATIO) {
    for (size_t c = 0; c * CW < n; ++c) {
      const size_t m = std::min(CW, n - c * CW);
      cl.raw.emplace_back(in + c * CW * wb, in + (c * CW + m) * wb);
      cl.words.push_back(m);
    }
    return cl;
  }
  std::vector<uint64_t> x(n), V(n), Dist(n);
  std::vector<uint32_t> h(n);
  for (size_t i = 0; i < n; ++i) x[i] = load_le<uint64_t>(in + 8 * i);
  fcm_hash(x.data(), n, h.data());
  fcm_match(x.data(), h.data(), n, V.data(), Dist.data());
  for (size_t t = 0; t * 2048 < n; ++t) {
    const size_t m = std::min<size_t>(2048, n - t * 2048);
    for (const std::vector<uint64_t>* arr : {&V, &Dist}) {
      Bytes b(8 * m);
      for (size_t i = 0; i < m; ++i) store_le<uint64_t>(b.data() + 8 * i, (*arr)[t * 2048 + i]);
      cl.raw.push_back(std::move(b));
      cl.words.push_back(m);
    }
  }
  return cl;
}

size_t chunk_count(int algo, size_t in_bytes) {
  const size_t wb = word_bytes_of(algo), n = in_bytes / wb;
  if (algo == DPRATIO) return 2 * ceil_div(n, 2048);
  return ceil_div(n, 16384 / wb);
}

bool valid_algo(int algo) { return algo >= SPSPEED && algo <= DPRATIO; }

}  // namespace

extern "C" {

size_t lcfo_max_compressed_size(int algo, size_t in_bytes) {
  if (!valid_algo(algo)) return 0;
  const size_t wb = word_bytes_of(algo), n = in_bytes / wb;
  const size_t C = chunk_count(algo, in_bytes);
  size_t total = round_up(32 + 4 * C, 16);
  if (algo == DPRATIO) {
    for (size_t t = 0; t * 2048 < n; ++t) total += 2 * round_up(8 * std::min<size_t>(2048, n - t * 2048), 16);
  } else {
    const size_t CW = 16384 / wb;
    for (size_t c = 0; c < C; ++c) total += round_up(wb * std::min(CW, n - c * CW), 16);
  }
  return total;
}

int lcfo_compress(int algo, const uint8_t* in, size_t in_bytes, uint8_t* out,
                  size_t out_capacity, size_t* out_bytes) {
  if (!valid_algo(algo)) return E_ARG;
  const size_t wb = word_bytes_of(algo);
  if (in_bytes % wb) return E_ARG;
  if (out_capacity < lcfo_max_compressed_size(algo, in_bytes)) return E_SMALL;
  ChunkList cl = make_chunks(algo, in, in_bytes);
  const size_t C = cl.raw.size();
  const size_t base = round_up(32 + 4 * C, 16);
  std::memset(out, 0, base);
  size_t off = base;
  for (size_t c = 0; c < C; ++c) {
    Bytes enc = encode_chunk(algo, cl.raw[c].data(), cl.words[c]);
    uint32_t entry;
    const Bytes* src = &enc;
    if (enc.size() >= cl.raw[c].size()) {  // raw fallback (L104), ties → raw
      src = &cl.raw[c];
      entry = (uint32_t)src->size() | 0x80000000u;
    } else {
      entry = (uint32_t)enc.size();
    }
    store_le<uint32_t>(out + 32 + 4 * c, entry);
    std::memcpy(out + off, src->data(), src->size());
    std::memset(out + off + src->size(), 0, round_up(src->size(), 16) - src->size());
    off += round_up(src->size(), 16);
  }
  store_le<uint32_t>(out + 0, 0x3146434Cu);
  out[4] = 1;
  out[5] = (uint8_t)algo;
  out[6] = (uint8_t)wb;
  out[7] = 0;
  store_le<uint64_t>(out + 8, in_bytes);
  store_le<uint64_t>(out + 16, C);
  store_le<uint64_t>(out + 24, off - base);
  if (out_bytes) *out_bytes = off;
  return OK;
}

int lcfo_decompress(int algo, const uint8_t* in, size_t in_bytes, uint8_t* out,
                    size_t out_capacity, size_t* out_bytes) {
  if (!valid_algo(algo)) return E_ARG;
  if (in_bytes < 32) return E_CORRUPT;
  const size_t wb = word_bytes_of(algo);
  if (load_le<uint32_t>(in) != 0x3146434Cu || in[4] != 1 || in[7] != 0) return E_CORRUPT;
  if (in[5] > 3) return E_CORRUPT;
  if (in[5] != algo) return E_DTYPE;
  if (in[6] != wb) return E_CORRUPT;
  const uint64_t nb = load_le<uint64_t>(in + 8), C = load_le<uint64_t>(in + 16),
                 pb = load_le<uint64_t>(in + 24);
  if (nb % wb || C != chunk_count(algo, nb)) return E_CORRUPT;
  if (C > (in_bytes - 32) / 4) return E_CORRUPT;
  const size_t base = round_up(32 + 4 * C, 16);
  if (base > in_bytes || pb > in_bytes - base) return E_CORRUPT;
  if (out_capacity < nb) return E_SMALL;
  const size_t n = nb / wb;
  std::vector<uint64_t> V, Dist;
  if (algo == DPRATIO) { V.assign(n, 0); Dist.assign(n, 0); }
  size_t off = 0;
  for (size_t c = 0; c < C; ++c) {
    const uint32_t entry = load_le<uint32_t>(in + 32 + 4 * c);
    const size_t len = entry & 0x7FFFFFFFu;
    const bool raw = entry >> 31;
    size_t first_word, m;
    if (algo == DPRATIO) {
      first_word = (c / 2) * 2048;
      m = std::min<size_t>(2048, n - first_word);
    } else {
      first_word = c * (16384 / wb);
      m = std::min<size_t>(16384 / wb, n - first_word);
    }
    if (off + round_up(len, 16) > pb) return E_CORRUPT;
    const uint8_t* src = in + base + off;
    uint8_t* dst = (algo == DPRATIO)
                       ? reinterpret_cast<uint8_t*>(((c & 1) ? Dist : V).data() + first_word)
                       : out + first_word * wb;
    std::vector<uint8_t> tmp(m * wb);
    if (raw) {
      if (len != m * wb) return E_CORRUPT;
      std::memcpy(tmp.data(), src, len);
    } else {
      if (len >= m * wb) return E_CORRUPT;
      if (int st = decode_chunk(algo, src, len, m, tmp.data())) return st;
    }
    if (algo == DPRATIO) {
      for (size_t i = 0; i < m; ++i) ((c & 1) ? Dist : V)[first_word + i] = load_le<uint64_t>(tmp.data() + 8 * i);
    } else {
      std::memcpy(dst, tmp.data(), m * wb);
    }
    off += round_up(len, 16);
  }
  if (off != pb) return E_CORRUPT;
  if (algo == DPRATIO) {
    std::vector<uint64_t> x(n);
    if (int st = fcm_dec(V.data(), Dist.data(), n, x.data())) return st;
    for (size_t i = 0; i < n; ++i) store_le<uint64_t>(out + 8 * i, x[i]);
  }
  if (out_bytes) *out_bytes = nb;
  return OK;
}

int lcfo_compress_chunks(int algo, const uint8_t* in, size_t in_bytes, uint64_t first_chunk,
                         uint64_t n_chunks, uint32_t* table, uint8_t* payload,
                         size_t payload_capacity, uint64_t* payload_bytes) {
  if (!valid_algo(algo) || algo == DPRATIO) return E_ARG;
  const size_t wb = word_bytes_of(algo);
  if (in_bytes % wb) return E_ARG;
  const size_t C = chunk_count(algo, in_bytes), n = in_bytes / wb, CW = 16384 / wb;
  if (first_chunk > C || n_chunks > C - first_chunk) return E_ARG;
  size_t off = 0;
  for (uint64_t c = first_chunk; c < first_chunk + n_chunks; ++c) {
    const size_t m = std::min(CW, n - c * CW);
    const uint8_t* raw = in + c * CW * wb;
    Bytes enc = encode_chunk(algo, raw, m);
    Bytes rawv(raw, raw + m * wb);
    const bool is_raw = enc.size() >= rawv.size();
    const Bytes& src = is_raw ? rawv : enc;
    if (off + round_up(src.size(), 16) > payload_capacity) return E_SMALL;
    table[c - first_chunk] = (uint32_t)src.size() | (is_raw ? 0x80000000u : 0u);
    std::memcpy(payload + off, src.data(), src.size());
    std::memset(payload + off + src.size(), 0, round_up(src.size(), 16) - src.size());
    off += round_up(src.size(), 16);
  }
  *payload_bytes = off;
  return OK;
}

void lcfo_diffms32_enc(const uint32_t* x, size_t n, uint32_t* u) { diffms_enc<uint32_t>(x, n, u); }
void lcfo_diffms32_dec(const uint32_t* u, size_t n, uint32_t* x) { diffms_dec<uint32_t>(u, n, x); }
void lcfo_diffms64_enc(const uint64_t* x, size_t n, uint64_t* u) { diffms_enc<uint64_t>(x, n, u); }
void lcfo_diffms64_dec(const uint64_t* u, size_t n, uint64_t* x) { diffms_dec<uint64_t>(u, n, x); }

size_t lcfo_mplg32_enc(const uint32_t* u, size_t n, uint8_t* out) {
  Bytes b = mplg_enc<uint32_t>(u, n);
  std::memcpy(out, b.data(), b.size());
  return b.size();
}
int lcfo_mplg32_dec(const uint8_t* in, size_t len, size_t n, uint32_t* u) {
  return mplg_dec<uint32_t>(in, len, n, u);
}
size_t lcfo_mplg64_enc(const uint64_t* u, size_t n, uint8_t* out) {
  Bytes b = mplg_enc<uint64_t>(u, n);
  std::memcpy(out, b.data(), b.size());
  return b.size();
}
int lcfo_mplg64_dec(const uint8_t* in, size_t len, size_t n, uint64_t* u) {
  return mplg_dec<uint64_t>(in, len, n, u);
}
void lcfo_bit32_enc(const uint32_t* u, size_t n, uint32_t* t) { bit32_enc(u, n, t); }
void lcfo_bit32_dec(const uint32_t* t, size_t n, uint32_t* u) { bit32_dec(t, n, u); }
size_t lcfo_rze_enc(const uint8_t* d, size_t L, uint8_t* out) {
  Bytes b = rze_enc(d, L);
  std::memcpy(out, b.data(), b.size());
  return b.size();
}
int lcfo_rze_dec(const uint8_t* in, size_t len, size_t L, uint8_t* d) { return rze_dec(in, len, L, d); }
void lcfo_fcm_hash(const uint64_t* x, size_t n, uint32_t* h) { fcm_hash(x, n, h); }
void lcfo_fcm_match(const uint64_t* x, const uint32_t* h, size_t n, uint64_t* V, uint64_t* Dist) {
  fcm_match(x, h, n, V, Dist);
}
int lcfo_fcm_dec(const uint64_t* V, const uint64_t* Dist, size_t n, uint64_t* x) {
  return fcm_dec(V, Dist, n, x);
}
size_t lcfo_raze_enc(const uint8_t* in, size_t L, uint8_t* out) {
  Bytes b = adaptive_enc(in, L, false);
  std::memcpy(out, b.data(), b.size());
  return b.size();
}
size_t lcfo_rare_enc(const uint8_t* in, size_t L, uint8_t* out) {
  Bytes b = adaptive_enc(in, L, true);
  std::memcpy(out, b.data(), b.size());
  return b.size();
}
static int adaptive_dec_c(const uint8_t* in, size_t len, bool rare, uint8_t* out, size_t cap, size_t* L) {
  Bytes b;
  if (int st = adaptive_dec(in, len, rare, b)) return st;
  if (b.size() > cap) return E_SMALL;
  std::memcpy(out, b.data(), b.size());
  *L = b.size();
  return OK;
}
int lcfo_raze_dec(const uint8_t* in, size_t len, uint8_t* out, size_t cap, size_t* L) {
  return adaptive_dec_c(in, len, false, out, cap, L);
}
int lcfo_rare_dec(const uint8_t* in, size_t len, uint8_t* out, size_t cap, size_t* L) {
  return adaptive_dec_c(in, len, true, out, cap, L);
}

}  // extern "C"
