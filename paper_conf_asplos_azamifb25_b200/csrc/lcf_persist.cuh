// lcf_persist.cuh — the warp roles shared by the persistent chunk kernels:
//   enc_loader  : ticket → 1-D TMA bulk load of a raw chunk into an input ring
//   enc_storer  : decoupled look-back (L122) → TMA bulk store of the encoded
//                 chunk → size-table entry; last chunk writes the header
//   dec_loader  : batched tickets → size entries → aggregates published at once
//                 → one look-back per batch → TMA bulk loads of the payloads
// The shared-memory struct `Sm` provides the ring buffers and mbarriers
// (in/full_in/empty_in/in_chunk for encoders; out/full_out/empty_out/out_chunk/
// out_len/out_raw for storers; in/full_in/empty_in/chunk/len/flags for decoders).
#pragma once
#include "lcf_kernels.cuh"
#include "lcf_pipe.cuh"

namespace lcf {

constexpr uint64_t kNoChunk = ~0ull;

__device__ __forceinline__ uint32_t chunk_words(uint64_t n_words_total, uint64_t gc, uint32_t CW) {
  return (uint32_t)umin64((uint64_t)CW, n_words_total - gc * CW);
}

// Ticket dispenser: ticket[0] counts handed-out tickets, ticket[1] counts CTAs
// that drew their final (failing) ticket; the last one resets both for the
// next launch on the stream.
__device__ __forceinline__ void ticket_retire(const LaunchCtx& ctx) {
  if (atomicAdd(ctx.ticket + 1, 1ull) == gridDim.x - 1) {
    ctx.ticket[0] = 0;
    ctx.ticket[1] = 0;
  }
}

template <int NS, class Sm>
__device__ __forceinline__ void enc_loader(Sm& S, const EncArgs& a, const LaunchCtx& ctx, uint32_t lane,
                                           uint32_t wb) {
  const uint32_t CW = kChunkBytes / wb;
  for (uint32_t it = 0;; ++it) {
    const uint32_t s = it % NS, ph = (it / NS) & 1;
    mbar_wait(&S.empty_in[s], ph ^ 1);
    uint64_t t = 0;
    if (lane == 0) t = atomicAdd(ctx.ticket, 1ull);
    t = __shfl_sync(0xFFFFFFFFu, t, 0);
    if (t >= a.n_chunks) {
      if (lane == 0) {
        S.in_chunk[s] = kNoChunk;
        mbar_arrive(&S.full_in[s]);
        ticket_retire(ctx);
      }
      return;
    }
    const uint32_t bytes = chunk_words(a.n_words_total, a.first_chunk + t, CW) * wb;
    const uint8_t* src = reinterpret_cast<const uint8_t*>(a.in) + t * kChunkBytes;
    if (lane == 0) trace_stamp(a, t, 0);
    if ((bytes & 15) == 0) {
      if (lane == 0) {
        S.in_chunk[s] = t;
        mbar_arrive_expect_tx(&S.full_in[s], bytes);
        tma_load_1d(S.in[s], src, bytes, &S.full_in[s]);
      }
    } else {  // ragged tail chunk: plain loads
      for (uint32_t i = lane; i < bytes / 4; i += 32) S.in[s][i] = reinterpret_cast<const uint32_t*>(src)[i];
      if (lane == 0) S.in_chunk[s] = t;
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.full_in[s]);
    }
  }
}

// kInPlace: the compute warps encode into the chunk's own input stage (S.in),
// and the storer hands that stage back to the loader (S.empty_in) once the TMA
// unit has read it — no separate output ring.
// kZeroOut: the storer re-zeroes the stored bytes of an output slot before it
// hands the slot back (the compute warps OR bit fields into a zeroed slot).
template <int NO, int NSTORERS, class Sm, bool kInPlace = false, bool kZeroOut = false>
__device__ __forceinline__ void enc_storer(Sm& S, const EncArgs& a, const LaunchCtx& ctx, uint32_t lane,
                                           uint32_t first) {
  for (uint32_t it = first;; it += NSTORERS) {
    const uint32_t o = it % NO, ph = (it / NO) & 1;
    mbar_wait(&S.full_out[o], ph);
    const uint64_t t = S.out_chunk[o];
    if (t == kNoChunk) break;
    const uint32_t len = S.out_len[o], raw = S.out_raw[o];
    if (lane == 0) trace_stamp(a, t, 5);
    const uint64_t excl = lookback_warp(ctx, t, round16(len));
    if (lane == 0) trace_stamp(a, t, 6);
    if (lane == 0) {
      const void* buf;
      if constexpr (kInPlace) buf = S.in[o];
      else buf = S.out[o];
      tma_store_1d(a.payload + excl, buf, (uint32_t)round16(len));
      tma_store_commit();
      a.table[t] = len | (raw ? kRawFlag : 0u);
      if (t == a.n_chunks - 1) finish_encode(a, excl + round16(len));
      if (t == 0)
        for (uint32_t i = 0; i < a.pad_len; ++i) a.pad_start[i] = 0;
      tma_store_wait_read0();  // the slot's bytes have been read by the TMA unit
      trace_stamp(a, t, 7);
      if constexpr (!kZeroOut) {
        if constexpr (kInPlace) mbar_arrive(&S.empty_in[o]);
        else mbar_arrive(&S.empty_out[o]);
      }
    }
    __syncwarp();
    if constexpr (kZeroOut) {
      uint4* z = reinterpret_cast<uint4*>(S.out[o]);
      for (uint32_t j = lane; j < round16(len) / 16; j += 32) z[j] = make_uint4(0, 0, 0, 0);
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.empty_out[o]);
    }
  }
  if (lane == 0) tma_store_wait_all0();
}

// Compute-warp side of the end marker: forward kNoChunk to every storer.
template <int NO, int NSTORERS, class Sm>
__device__ __forceinline__ void enc_forward_end(Sm& S, uint32_t it, uint32_t cw, uint32_t lane) {
  for (uint32_t j = 0; j < NSTORERS; ++j) {
    const uint32_t oj = (it + j) % NO, phj = ((it + j) / NO) & 1;
    mbar_wait(&S.empty_out[oj], phj ^ 1);
    if (cw == 0 && lane == 0) S.out_chunk[oj] = kNoChunk;
    __syncwarp();
    if (lane == 0) mbar_arrive(&S.full_out[oj]);
  }
}

// Decoder loader for chunk-per-CW-words streams (SPspeed, SPratio, DPspeed).
template <int NS, int BATCH, class Sm>
__device__ __forceinline__ void dec_loader(Sm& S, const DecArgs& a, const LaunchCtx& ctx, uint32_t lane,
                                           uint32_t wb) {
  const uint32_t CW = kChunkBytes / wb;
  uint64_t n_words = 0, n_chunks = 0, base = 0, payload = 0;
  const bool hdr_ok = read_header(a, ctx, n_words, n_chunks, base, payload);
  const bool small = hdr_ok && n_words * wb > a.out_capacity;
  uint32_t it = 0;
  for (;;) {
    // a ticket claims BATCH consecutive chunks: one look-back per batch, the
    // batch's own offsets from its size-table entries
    uint64_t tb = 0;
    if (lane == 0) tb = atomicAdd(ctx.ticket, 1ull);
    tb = __shfl_sync(0xFFFFFFFFu, tb, 0) * BATCH;
    if (!hdr_ok || small || tb >= n_chunks) {
      const uint32_t s = it % NS, ph = (it / NS) & 1;
      mbar_wait(&S.empty_in[s], ph ^ 1);
      if (lane == 0) {
        if (tb == 0 && !hdr_ok) record_error(ctx, DERR_CORRUPT);
        if (tb == 0 && small) record_error(ctx, DERR_SMALL);
        S.chunk[s] = kNoChunk;
        mbar_arrive(&S.full_in[s]);
        ticket_retire(ctx);
      }
      return;
    }
    const uint32_t nb = (uint32_t)umin64(BATCH, n_chunks - tb);
    const uint64_t t = tb + lane;
    uint32_t len = 0, raw = 0;
    bool bad = false;
    if (lane < nb) {
      const uint32_t e = reinterpret_cast<const uint32_t*>(a.stream + kHeaderBytes)[t];
      len = e & ~kRawFlag;
      raw = e >> 31;
      const uint32_t m = chunk_words(n_words, t, CW);
      bad = raw ? len != m * wb : len >= m * wb;
      lookback_publish(ctx, t, bad ? 0 : round16(len));
    }
    const uint64_t agg = (lane < nb && !bad) ? round16(len) : 0;
    uint64_t x = agg;  // exclusive prefix inside the batch
#pragma unroll
    for (int d = 1; d < BATCH; d <<= 1) {
      const uint64_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
      if ((int)lane >= d) x += y;
    }
    x -= agg;
    const uint64_t base_b = lookback_warp(ctx, tb, __shfl_sync(0xFFFFFFFFu, agg, 0));
    const uint64_t excl = base_b + x;
    if (lane > 0 && lane < nb) st_relaxed_u64(ctx.status + t, make_status(kFlagInc, ctx.epoch, excl + agg));
    const uint64_t end = excl + round16(len);
    if (lane < nb && !bad && (end > payload || (t == n_chunks - 1 && end != payload))) bad = true;
    for (uint32_t j = 0; j < nb; ++j, ++it) {
      const uint32_t s = it % NS, ph = (it / NS) & 1;
      const uint32_t lj = __shfl_sync(0xFFFFFFFFu, len, j), rj = __shfl_sync(0xFFFFFFFFu, raw, j);
      const bool bj = __shfl_sync(0xFFFFFFFFu, bad, j);
      const uint64_t ej = __shfl_sync(0xFFFFFFFFu, excl, j);
      mbar_wait(&S.empty_in[s], ph ^ 1);
      if (lane == 0) {
        if (bj) record_error(ctx, DERR_CORRUPT);
        S.chunk[s] = tb + j;
        S.len[s] = lj;
        S.flags[s] = rj | (bj ? 2u : 0u);
        if (!bj && lj) {
          mbar_arrive_expect_tx(&S.full_in[s], (uint32_t)round16(lj));
          tma_load_1d(S.in[s], a.stream + base + ej, (uint32_t)round16(lj), &S.full_in[s]);
        } else {
          mbar_arrive(&S.full_in[s]);
        }
      }
    }
  }
}

}  // namespace lcf
