/*
 * lcf_oracle.h — plain, slow, single-threaded CPU oracle for the four LC-style
 * floating-point codecs of Azami, Fallin & Burtscher, "Efficient Lossless
 * Compression of Scientific Floating-Point Data on CPUs and GPUs", ASPLOS '25
 * (PAPER.md). Stream format: FORMAT.md.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant with the CUDA path
 * (paper_conf_asplos_azamifb25_b200/csrc), and neither includes the other.
 *
 * Every function follows the passage it cites step by step; no blocking,
 * fusion or reordering. Parity status of each function: DESIGN.md §4.
 *
 * Status codes mirror lcf_status_t by value (FORMAT.md does not need them):
 *   0 success, 1 invalid argument, 2 dtype mismatch, 3 buffer too small,
 *   4 corrupt stream.
 */
#ifndef LCF_ORACLE_H
#define LCF_ORACLE_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- whole streams (FORMAT.md §1–§2) ------------------------------------ */
/* algo: 0 SPspeed, 1 SPratio, 2 DPspeed, 3 DPratio. */
size_t lcfo_max_compressed_size(int algo, size_t in_bytes);
int lcfo_compress(int algo, const uint8_t* in, size_t in_bytes,
                  uint8_t* out, size_t out_capacity, size_t* out_bytes);
int lcfo_decompress(int algo, const uint8_t* in, size_t in_bytes,
                    uint8_t* out, size_t out_capacity, size_t* out_bytes);
/* Chunk range [first_chunk, first_chunk+n_chunks) of the stream for the whole
 * input `in` (in_bytes): writes the n_chunks size-table entries and the chunks'
 * padded payloads (offsets relative to the first of them). DPratio: rejected
 * (FCM is a whole-array pass). */
int lcfo_compress_chunks(int algo, const uint8_t* in, size_t in_bytes,
                         uint64_t first_chunk, uint64_t n_chunks,
                         uint32_t* table, uint8_t* payload, size_t payload_capacity,
                         uint64_t* payload_bytes);

/* ---- single stages (FORMAT.md §3–§6) ------------------------------------ */
void lcfo_diffms32_enc(const uint32_t* x, size_t n, uint32_t* u);
void lcfo_diffms32_dec(const uint32_t* u, size_t n, uint32_t* x);
void lcfo_diffms64_enc(const uint64_t* x, size_t n, uint64_t* u);
void lcfo_diffms64_dec(const uint64_t* u, size_t n, uint64_t* x);
/* MPLG: returns encoded length; out must hold lcfo_max_compressed_size-like
 * room (n·W/8 + 64 bytes suffices). dec returns status. */
size_t lcfo_mplg32_enc(const uint32_t* u, size_t n, uint8_t* out);
int lcfo_mplg32_dec(const uint8_t* in, size_t len, size_t n, uint32_t* u);
size_t lcfo_mplg64_enc(const uint64_t* u, size_t n, uint8_t* out);
int lcfo_mplg64_dec(const uint8_t* in, size_t len, size_t n, uint64_t* u);
void lcfo_bit32_enc(const uint32_t* u, size_t n, uint32_t* t);
void lcfo_bit32_dec(const uint32_t* t, size_t n, uint32_t* u);
/* RZE on L bytes: out needs L + L/4 + 8 bytes. */
size_t lcfo_rze_enc(const uint8_t* d, size_t L, uint8_t* out);
int lcfo_rze_dec(const uint8_t* in, size_t len, size_t L, uint8_t* d);
/* FCM (whole array). h: 20-bit hashes, one per word. */
void lcfo_fcm_hash(const uint64_t* x, size_t n, uint32_t* h);
void lcfo_fcm_match(const uint64_t* x, const uint32_t* h, size_t n,
                    uint64_t* V, uint64_t* Dist);
int lcfo_fcm_dec(const uint64_t* V, const uint64_t* Dist, size_t n, uint64_t* x);
/* RAZE / RARE on L < 65536 bytes: out needs L + 3 bytes. */
size_t lcfo_raze_enc(const uint8_t* in, size_t L, uint8_t* out);
int lcfo_raze_dec(const uint8_t* in, size_t len, uint8_t* out, size_t cap, size_t* L);
size_t lcfo_rare_enc(const uint8_t* in, size_t L, uint8_t* out);
int lcfo_rare_dec(const uint8_t* in, size_t len, uint8_t* out, size_t cap, size_t* L);

#ifdef __cplusplus
}
#endif
#endif
