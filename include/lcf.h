/*
 * lcf.h — C ABI of liblcf.so, the B200 (sm_100a) implementation of the four
 * lossless floating-point codecs of Azami, Fallin & Burtscher, ASPLOS '25
 * (PAPER.md; "L<n>" = PAPER.md line). Stream format: FORMAT.md (LCF1).
 *
 * Problem statement (L41, L92, L278, L354): losslessly compress an array of
 * IEEE-754 float32 (SPspeed, SPratio) or float64 (DPspeed, DPratio) values,
 * treated bit-for-bit as integers, into ONE contiguous compressed block whose
 * chunks are placed by a prefix sum of their sizes (L120–122), and decompress
 * it again; the stream is a pure function of the input (L415) and identical to
 * the CPU oracle's.
 *
 * Conventions (all entry points):
 *  - Pointers named d_* are DEVICE pointers on the current CUDA device, owned by
 *    the caller; the library never frees or retains them beyond the stream work
 *    it enqueues. h_* pointers are HOST pointers (pinned memory recommended).
 *  - Calls are stream-ordered and asynchronous on `stream` (a cudaStream_t;
 *    NULL = legacy default stream) unless an `out_bytes` pointer is non-NULL, in
 *    which case the call synchronises `stream` to report the size.
 *  - Library-owned scratch (ticket counter, look-back status, FCM sort buffers,
 *    error word) is cached per (device, stream) and grown on demand; the first
 *    call for a (device, stream, size) may allocate.
 *  - Errors: arguments are validated on the host before anything is enqueued.
 *    Stream corruption found by decoder kernels is recorded on the device and
 *    reported as LCF_ERROR_CORRUPT_STREAM by the next synchronising call on that
 *    stream (out_bytes != NULL, lcf_get_info, lcf_check_stream). Decoders never
 *    read or write outside [d_in, d_in+in_bytes) and [d_out, d_out+out_capacity).
 *  - There is no CPU fallback: with no usable CUDA device every call returns
 *    LCF_ERROR_CUDA.
 */
#ifndef LCF_H
#define LCF_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum { LCF_SPSPEED = 0, LCF_SPRATIO = 1, LCF_DPSPEED = 2, LCF_DPRATIO = 3 } lcf_algo_t;
typedef enum { LCF_FLOAT32 = 0, LCF_FLOAT64 = 1 } lcf_dtype_t;
typedef enum {
  LCF_SUCCESS = 0,
  LCF_ERROR_INVALID_ARGUMENT = 1,
  LCF_ERROR_DTYPE_MISMATCH = 2,
  LCF_ERROR_BUFFER_TOO_SMALL = 3,
  LCF_ERROR_CORRUPT_STREAM = 4,
  LCF_ERROR_CUDA = 5,
  LCF_ERROR_OUT_OF_MEMORY = 6
} lcf_status_t;

/* Worst-case stream size for in_bytes of input (pure host function):
 * round16(32 + 4·C) + Σ_c round16(raw bytes of chunk c) — every chunk stored raw
 * (L104). DPratio's FCM doubles the data (L185), so its bound is ≈ 2·in_bytes.
 * Returns 0 for an invalid algo. */
size_t lcf_max_compressed_size(lcf_algo_t algo, lcf_dtype_t dtype, size_t in_bytes);

/* Compress in_bytes of float words at d_in into the LCF1 stream at d_out.
 * in_bytes must be a multiple of the word size (4 or 8) → else INVALID_ARGUMENT;
 * SP codecs need LCF_FLOAT32 and DP codecs LCF_FLOAT64 → else DTYPE_MISMATCH
 * (L41); out_capacity ≥ lcf_max_compressed_size(...) → else BUFFER_TOO_SMALL.
 * d_in must be 16-byte aligned. in_bytes = 0 yields the 32-byte header.
 * DPratio only: fewer than 2^31 words (16 GiB) per call → else INVALID_ARGUMENT
 * (its FCM sort records carry a 32-bit word index; the oracle has no such
 * limit; larger arrays go through the sharded calls below, whose shards each
 * stay under it).
 * Stages per 16 KiB chunk: SPspeed DIFFMS→MPLG (L108–118), SPratio
 * DIFFMS→BIT→RZE (L138–158), DPspeed DIFFMS→MPLG, DPratio FCM→DIFFMS→RAZE→RARE
 * (L168–201); raw fallback per chunk (L104); placement by a single-pass
 * decoupled look-back over chunk sizes (L122). *out_bytes (if non-NULL)
 * receives the stream length after a stream synchronisation. */
lcf_status_t lcf_compress(lcf_algo_t algo, lcf_dtype_t dtype, const void* d_in, size_t in_bytes,
                          void* d_out, size_t out_capacity, size_t* out_bytes, void* stream);

/* Decompress the LCF1 stream of in_bytes at d_in into d_out (16-byte aligned).
 * With out_bytes == NULL nothing is read back: the header, size table and
 * payloads are validated by the kernels themselves (no host round trip), and an
 * out_capacity smaller than the stream's n_bytes or a malformed stream is
 * recorded on the device and reported by the next synchronising call. With
 * out_bytes != NULL the header is first read to the host (one 32-byte D2H) and
 * checked there, returning CORRUPT_STREAM / DTYPE_MISMATCH / BUFFER_TOO_SMALL
 * directly, and device-found corruption is reported before returning.
 * Inverse stages in reverse order (L94); chunk read offsets from the prefix sum
 * of stored sizes (L120). `stream` is a cudaStream_t passed as void*. */
lcf_status_t lcf_decompress(lcf_algo_t algo, lcf_dtype_t dtype, const void* d_in, size_t in_bytes,
                            void* d_out, size_t out_capacity, size_t* out_bytes, void* stream);

/* Synchronise `stream` and read the 32-byte header at d_in (D2H): any of the
 * out-pointers may be NULL. Returns CORRUPT_STREAM for a malformed header. */
lcf_status_t lcf_get_info(const void* d_in, size_t in_bytes, lcf_algo_t* algo, lcf_dtype_t* dtype,
                          size_t* uncompressed_bytes, size_t* compressed_bytes, void* stream);

/* Synchronise `stream`; returns CORRUPT_STREAM (or BUFFER_TOO_SMALL) if any
 * decompression enqueued on it since the previous check found a malformed
 * stream, else SUCCESS. */
lcf_status_t lcf_check_stream(void* stream);

/* ---- host-buffer convenience (the end-to-end path) ----------------------
 * Same as lcf_compress / lcf_decompress but h_in and h_out are HOST buffers:
 * the library copies h_in to device scratch, runs the codec on `stream`, copies
 * the result back and synchronises. *out_bytes is always written.
 * SPspeed, SPratio and DPspeed inputs larger than one slice (~1/8 of the input,
 * 4..64 MiB; env LCF_HOST_SLICE_BYTES overrides) are pipelined: chunk
 * encodings are context-free, so each slice is coded as its
 * own sub-stream while the next slice's host→device copy and the previous
 * slice's device→host copy run on two library-owned streams; the host stitches
 * the same bytes lcf_compress writes (FORMAT.md). Pinned host buffers let the
 * two copy directions overlap. compress: out_capacity must hold the stitched
 * stream (BUFFER_TOO_SMALL otherwise; lcf_max_compressed_size always does).
 * decompress: the header and size table are read on the host; any malformed
 * slice reports CORRUPT_STREAM. DPratio decompression streams by tile ranges
 * (distances into earlier slices read their final output); DPratio
 * compression by tile slices carrying the FCM state of the earlier slices (the
 * sharded-DPratio calls below): the same bytes as lcf_compress. */
lcf_status_t lcf_compress_host(lcf_algo_t algo, lcf_dtype_t dtype, const void* h_in, size_t in_bytes,
                               void* h_out, size_t out_capacity, size_t* out_bytes, void* stream);
lcf_status_t lcf_decompress_host(lcf_algo_t algo, lcf_dtype_t dtype, const void* h_in, size_t in_bytes,
                                 void* h_out, size_t out_capacity, size_t* out_bytes, void* stream);

/* ---- sharded mode (one process per GPU) ----------------------
 * Compress chunks [first_chunk, first_chunk + k) of the stream for an input of
 * total_in_bytes, where d_in_shard holds exactly those chunks' words
 * (shard_bytes). Writes the k size-table entries to d_table_slice (u32 each),
 * the chunks' padded payloads contiguously to d_payload (offsets from 0), and
 * the piece's payload byte count to the DEVICE u64 *d_payload_bytes (so it can
 * feed an NCCL all-gather on the same stream without a host sync). The
 * concatenation header ‖ table slices ‖ pad ‖ payload pieces, in chunk order, is
 * byte-identical to lcf_compress's stream. Not available for DPratio (its FCM
 * stage is a whole-array pass, L104): INVALID_ARGUMENT. */
lcf_status_t lcf_compress_shard(lcf_algo_t algo, lcf_dtype_t dtype, const void* d_in_shard,
                                size_t shard_bytes, size_t total_in_bytes, uint64_t first_chunk,
                                void* d_table_slice, void* d_payload, size_t payload_capacity,
                                uint64_t* d_payload_bytes, void* stream);

/* Number of chunks of a stream for in_bytes of input (FORMAT.md §2). */
uint64_t lcf_num_chunks(lcf_algo_t algo, size_t in_bytes);

/* Write the 32-byte stream header (FORMAT.md §1) and the zero pad between the
 * size table and the payload base to d_stream (which must have room for
 * round16(32 + 4·n_chunks) bytes); total_payload_bytes is a host value. */
lcf_status_t lcf_write_header(lcf_algo_t algo, lcf_dtype_t dtype, size_t total_in_bytes,
                              uint64_t total_payload_bytes, void* d_stream, void* stream);

/* ---- sharded DPratio -----------------------------------
 * FCM compares a word with the ≤ 4 nearest preceding words
 * of the same hash anywhere before it (L174), so a shard of the array needs,
 * per hash, the last ≤ 4 words before its first word. For shards of whole
 * 2048-word tiles, in array order:
 *  1. lcf_dpratio_shard_summary: the shard's summary — per hash, its last ≤ 4
 *     words (global index, value); lcf_dpratio_summary_bytes() bytes, device;
 *  2. every shard's summary is made readable by the others (CUDA IPC over
 *     NVLink: lcf_ipc_export / lcf_ipc_import below; on one device, plain
 *     pointers), after a barrier;
 *  3. lcf_dpratio_merge_summary_ptrs: shard g's carry from the summaries of
 *     shards 0 … g−1 (d_summaries: host array of g device pointers in shard
 *     order; count 0: an empty carry). Per hash it reads shard g−1's entries
 *     first and goes further back only while fewer than 4 are found, so it
 *     reads about one summary's worth, not g. lcf_dpratio_merge_summaries is
 *     the same over g summaries stored contiguously;
 *  4. lcf_dpratio_compress_shard: the shard's 2 chunks per tile with that carry
 *     (NULL for shard 0), written like lcf_compress_shard: size-table slice,
 *     payload piece from offset 0, device u64 payload byte count.
 * The pieces assemble with lcf_write_header into exactly the 1-GPU stream.
 * d_x points at the shard's first word (global index first_word, a multiple
 * of 2048); the min(3, first_word) words before it must be readable and hold
 * the array's words first_word − 3 … first_word − 1 (the hash context of the
 * shard's first words, L172): a caller holding only its shard places the
 * previous shard's last 3 words before it. shard_bytes is a multiple of
 * 16384 unless the shard ends the array. Errors as lcf_compress_shard.
 * lcf_dpratio_compress_shard right after lcf_dpratio_shard_summary of the same
 * shard (same d_x, size, first_word) on the same stream reuses the summary's
 * sort of the shard; its words must not change in between.
 *
 * Decompression of a shard: d_in is the shard's own LCF1 sub-stream (header
 * for its words, its size-table slice, its payload piece), whose word 0 is
 * global word first_word. lcf_dpratio_decompress_shard decodes every tile and
 * follows FCM chains inside a tile (L197); a word whose distance leaves its
 * tile is read if that tile is already complete, else it is left PENDING:
 * d_out holds the global index of the word it copies and its bit in
 * d_pending is set. d_pending holds 2·ceil(n / 32) u32 words, n =
 * out_capacity / 8: the pending bitmap, then a bitmap marking the words that
 * pending words point at (the chain nodes, walked first by find_roots); the
 * call clears and writes both. Asynchronous; malformed input is reported by
 * lcf_check_stream. The pending words are then resolved over all shards, each
 * described by an lcf_dp_view (its words and bitmap — local pointers or
 * CUDA-IPC-mapped peer pointers; views sorted by first_word, contiguous from
 * word 0, ≤ 64 of them; `self` is the caller's shard, whose first_word is a
 * multiple of 32):
 *  a. every shard's lcf_dpratio_decompress_shard has completed (barrier);
 *  b. lcf_dpratio_find_roots(self): each pending word of shard `self` follows
 *     its chain through the views to the first word that is not pending (its
 *     root) and stores the root's global index (L197's union-find "find",
 *     with path compression; only ancestor indices are ever stored, so shards
 *     may run this concurrently);
 *  c. every shard's find_roots has completed (barrier);
 *  d. lcf_dpratio_gather_roots(self): each pending word of `self` takes its
 *     root's value and the bitmap is cleared.
 * After d on every shard (barrier), the words are final. A chain that points
 * forwards, or outside the views, is reported as CORRUPT_STREAM. */
typedef struct {
  uint64_t first_word;  /* global index of the view's word 0 */
  uint64_t n_words;     /* words in the view */
  void* d_words;        /* its decoded words (u64), device */
  uint32_t* d_pending;  /* its 2·ceil(n_words / 32) bitmap words (see above), device */
} lcf_dp_view;
size_t lcf_dpratio_summary_bytes(void);
lcf_status_t lcf_dpratio_shard_summary(const void* d_x, size_t shard_bytes, size_t total_in_bytes, uint64_t first_word,
                                       void* d_summary, void* stream);
lcf_status_t lcf_dpratio_merge_summaries(const void* d_summaries, size_t count, void* d_carry, void* stream);
lcf_status_t lcf_dpratio_merge_summary_ptrs(const void* const* d_summaries, size_t count, void* d_carry,
                                            void* stream);
lcf_status_t lcf_dpratio_compress_shard(const void* d_x, size_t shard_bytes, size_t total_in_bytes,
                                        uint64_t first_word, const void* d_carry, void* d_table_slice,
                                        void* d_payload, size_t payload_capacity, uint64_t* d_payload_bytes,
                                        void* stream);
lcf_status_t lcf_dpratio_decompress_shard(const void* d_in, size_t in_bytes, uint64_t first_word, void* d_out,
                                          size_t out_capacity, uint32_t* d_pending, void* stream);
lcf_status_t lcf_dpratio_find_roots(const lcf_dp_view* views, size_t count, size_t self, void* stream);
lcf_status_t lcf_dpratio_gather_roots(const lcf_dp_view* views, size_t count, size_t self, void* stream);

/* CUDA IPC plumbing for the sharded modes (one process per GPU on one node):
 * lcf_ipc_export writes a 64-byte handle of the device allocation holding
 * d_ptr and d_ptr's offset inside it; another process passes both to
 * lcf_ipc_import and gets a device pointer to the same bytes (over NVLink when
 * the GPUs differ), valid until lcf_ipc_close. A process cannot import its
 * own export (use its pointer). Errors: INVALID_ARGUMENT (null / unknown
 * pointer), CUDA (the driver refused). */
lcf_status_t lcf_ipc_export(const void* d_ptr, void* handle64, uint64_t* offset);
lcf_status_t lcf_ipc_import(const void* handle64, uint64_t offset, void** d_ptr);
lcf_status_t lcf_ipc_close(void* d_ptr);

/* Number of kernel launches the library enqueued since the process started
 * (bench/test accounting). */
uint64_t lcf_launch_count(void);

/* Kernel-time tracing. While enabled, the library brackets every kernel it
 * launches with a pair of CUDA events on the launching stream (CUB's sort
 * counts as one "kernel"). lcf_profile_report synchronises on the recorded
 * events, writes "name launches total_ms\n" per kernel into buf (NUL-terminated,
 * truncated to cap) and clears the record; it returns the untruncated length. */
void lcf_profile_enable(int enable);
size_t lcf_profile_report(char* buf, size_t cap);

#ifdef __cplusplus
}
#endif
#endif /* LCF_H */
