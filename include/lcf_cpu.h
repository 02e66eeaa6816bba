/*
 * lcf_cpu.h — C ABI of liblcf_cpu.so: the multi-threaded CPU codec of the four
 * codecs, bit-compatible with the B200 path (lcf.h) and
 * the oracle: same LCF1 stream (FORMAT.md), so a stream compressed on either
 * side decompresses on the other (the paper's CPU/GPU compatibility, L41, L354).
 *
 * This is the paper's CPU design (L104, L120), not a fallback of the GPU
 * library: liblcf.so never calls it and it never touches a GPU.
 *  - Compress: worker threads draw chunks from a dynamic worklist (an atomic
 *    counter, L104), encode a chunk into a private 16 KiB buffer, then wait
 *    (busy-wait with yield) until the previous chunk has published its end
 *    position, publish their own end (position + round16(len)) and copy the
 *    chunk into place (L120: "the write position … passed from chunk to chunk").
 *    DPratio first builds FCM's V and Dist arrays over the whole input (L104,
 *    L170–185): hash, a parallel stable LSD radix sort of (hash, index) on two
 *    10-bit digits, and the nearest-of-four match (A-14).
 *  - Decompress: the size table is prefix-summed (L120), then threads decode
 *    chunks from a worklist. DPratio then resolves FCM's distances tile by
 *    tile in index order (L197), a tile waiting on a flag of any earlier tile
 *    it references.
 *
 * Conventions: all pointers are HOST pointers owned by the caller; nothing is
 * retained after a call returns. n_threads ≤ 0 means
 * std::thread::hardware_concurrency(). Calls are synchronous and thread-safe
 * (no global state). Status codes are lcf.h's lcf_status_t values.
 */
#ifndef LCF_CPU_H
#define LCF_CPU_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* algo: 0 SPspeed, 1 SPratio, 2 DPspeed, 3 DPratio (lcf_algo_t);
 * dtype: 0 float32, 1 float64 (lcf_dtype_t). */

/* Worst-case stream size (same bound as lcf_max_compressed_size); 0 for an
 * invalid algo. */
size_t lcf_cpu_max_compressed_size(int algo, int dtype, size_t in_bytes);

/* Compress in_bytes of words at in into the LCF1 stream at out.
 * in_bytes not a multiple of the word size → 1 (INVALID_ARGUMENT); dtype not
 * the codec's → 2 (DTYPE_MISMATCH); out_capacity < lcf_cpu_max_compressed_size
 * → 3 (BUFFER_TOO_SMALL); allocation failure → 6. *out_bytes (may be NULL)
 * receives the stream length. Returns 0 on success. */
int lcf_cpu_compress(int algo, int dtype, const void* in, size_t in_bytes, void* out, size_t out_capacity,
                     size_t* out_bytes, int n_threads);

/* Decompress the LCF1 stream of in_bytes at in into out. A stream whose header
 * disagrees with algo → 4 (CORRUPT_STREAM), or with dtype → 2; out_capacity
 * below the stream's n_bytes → 3; any malformed chunk, size table or FCM
 * distance → 4. Never reads or writes outside [in, in+in_bytes) and
 * [out, out+out_capacity). *out_bytes (may be NULL) receives n_bytes. */
int lcf_cpu_decompress(int algo, int dtype, const void* in, size_t in_bytes, void* out, size_t out_capacity,
                       size_t* out_bytes, int n_threads);

#ifdef __cplusplus
}
#endif
#endif /* LCF_CPU_H */
