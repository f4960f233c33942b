/*
 * cszp2.h — C ABI of the B200-native cuSZp2 compressor (libcszp2.so).
 *
 * Implements the single-kernel error-bounded lossy compressor of
 *   Huang, Di, Li, Cappello, "cuSZp2: A GPU Lossy Compressor with Extreme
 *   Throughput and Optimized Compression Ratio", SC'24 (PAPER.md; P:n = line n)
 * for f32 / f64 fields on sm_100a. The stream format and the arithmetic
 * contract are FORMAT.md (repo root).
 *
 * Conventions for every entry point:
 *  - Plain pointers and sizes only; `stream` is a cudaStream_t passed as void*
 *    (NULL = legacy default stream). Pointers named d_* are DEVICE pointers,
 *    h_* are HOST pointers.
 *  - The caller owns every buffer; the library allocates nothing. Its only state
 *    is a per-(kernel, device) cache of launch attributes (dynamic shared-memory
 *    opt-in, resident-CTA count), so one process may drive several GPUs. Calls on
 *    different streams with disjoint buffers may run concurrently.
 *  - Work is enqueued on `stream` without host synchronisation, except where
 *    a function says it synchronises.
 *  - Return value: CSZP2_OK, or a synchronous error (bad argument, CUDA launch
 *    failure). Data-dependent failures are reported inside the stream header
 *    (status byte) and through d_status, never by the return value.
 *  - Alignment: d_in, d_out, d_cmp must be 16-byte aligned (TMA requirement);
 *    cudaMalloc'd pointers are.
 *  - Size: the 1D entry points take n <= 2^35 values (the dense side is a tensor of
 *    128-byte rows addressed by int32 TMA coordinates); larger n is ARG.
 */
#ifndef CSZP2_H
#define CSZP2_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* status / error codes */
#define CSZP2_OK 0
#define CSZP2_ERR_ARG 1    /* invalid argument (null pointer, dtype, mode, eb, alignment) */
#define CSZP2_ERR_CUDA 2   /* a CUDA call or kernel launch failed */
#define CSZP2_ERR_RANGE 3  /* stream status: a value's |x/2eb| exceeds 2^30-1 or is not finite (FORMAT.md §6.3) */
#define CSZP2_ERR_FORMAT 4 /* stream is not a valid FORMAT.md v1 stream for (n, dtype) */

/* dtype */
#define CSZP2_F32 0
#define CSZP2_F64 1
/* error-bound mode */
#define CSZP2_EB_ABS 0 /* |x - x'| <= eb                                   */
#define CSZP2_EB_REL 1 /* eb = lambda; |x - x'| <= lambda * (max - min)      */
/* lossless encoding mode */
#define CSZP2_ENC_PLAIN 0   /* Plain-FLE for every block (CUSZP2-P)                 */
#define CSZP2_ENC_OUTLIER 1 /* per-block Outlier-FLE when strictly smaller (CUSZP2-O) */

/* Decoded stream header (FORMAT.md §3). */
typedef struct {
    uint32_t magic;
    uint8_t version, dtype, enc_mode, log2L, eb_mode, status;
    uint16_t blocks_per_tile;
    uint64_t n;
    double eb;      /* as given by the caller (ABS bound or REL lambda) */
    double eb_abs;  /* bound used for quantization */
    uint64_t payload_bytes;
    uint64_t total_bytes;
} cszp2_header;

/* Bytes d_out of cszp2_compress must hold: the largest stream of n values
 * (FORMAT.md §2, roundup16(D + 128*nb)) plus 16 bytes of scratch used by the
 * kernel's tile ticket. Returns 0 for an invalid dtype. */
uint64_t cszp2_compress_bound(uint64_t n, int dtype);

/* Compression (P:84-102 problem statement; Fig 4 workflow ❶-❹).
 *  n           : number of values, 0 <= n <= 2^35 (TMA row coordinates are int32), else ARG.
 *  d_in        : n values of `dtype`, device, 16-byte aligned, read only.
 *  eb          : ABS bound, or REL lambda in (0,1); finite and > 0.
 *  d_out       : device buffer of cszp2_compress_bound(n, dtype) bytes,
 *                16-byte aligned; receives the stream (header first).
 *  d_out_bytes : nullable DEVICE uint64; receives the stream's total bytes
 *                (also in the header), so a multi-GPU caller can all-gather
 *                it without a host sync.
 * Enqueues: a zeroing kernel (header, tile index, ticket), the REL min/max kernel
 * (REL only), and the single fused compression kernel. */
int cszp2_compress(const void *d_in, uint64_t n, int dtype, double eb, int eb_mode,
                   int enc_mode, void *d_out, uint64_t *d_out_bytes, void *stream);

/* The two phases of cszp2_compress, exposed so callers (bench.py) can time
 * the dominant kernel alone. cszp2_compress == prepare then encode, with the
 * same arguments.
 * prepare: zero the header, tile index and ticket of d_out and, for REL, run the
 *   device min/max reduction that writes eb_abs into the header.
 * encode: zero the tile index (the lookback descriptors) and the ticket, then the
 *   fused kernel (❶ quantize, in-block difference, ❷ FLE, ❸ decoupled-lookback
 *   scan, ❹ concatenation). encode may be repeated on the same d_out (each call
 *   writes the whole stream again); with eb_mode REL it quantizes with the eb_abs
 *   the header holds, i.e. the one a preceding prepare (or prepare_range) on this
 *   d_out wrote, or a previous encode left there (the same value). REL encode
 *   on a d_out that never saw a prepare reads an undefined bound. */
int cszp2_compress_prepare(const void *d_in, uint64_t n, int dtype, double eb, int eb_mode,
                           void *d_out, void *stream);
int cszp2_compress_encode(const void *d_in, uint64_t n, int dtype, double eb, int eb_mode,
                          int enc_mode, void *d_out, uint64_t *d_out_bytes, void *stream);

/* Global REL for one field sharded across ranks (the paper's REL bound
 * is relative to the value range of the whole dataset). Per rank:
 *   cszp2_value_range(slab) -> reduce (min, max) across ranks (the caller's one
 *   16-byte collective) -> cszp2_compress_prepare_range(slab, lambda, range)
 *   -> cszp2_compress_encode(slab, lambda, CSZP2_EB_REL, ...).
 * The ranks' offset bytes and payloads then concatenate to the single-GPU stream's.
 * cszp2_value_range: d_work = 8 doubles (64 B, 16-byte aligned, device); on
 *   completion (stream-ordered) d_work[0] = min, d_work[1] = max over the non-NaN
 *   values of d_in, exact (T -> f64 conversions); (+inf, -inf) when there is none
 *   (n = 0 or all NaN). The other words are scratch. Errors: ARG, CUDA.
 * cszp2_compress_prepare_range: as cszp2_compress_prepare with eb_mode REL, except
 *   that eb_abs = eb * (max - min) comes from the device range d_range[0..1]
 *   (16-byte aligned) instead of a reduction over d_in; a zero or empty range gives
 *   eb_abs = eb, as for the local range (FORMAT.md §6.1). Errors as prepare. */
int cszp2_value_range(const void *d_in, uint64_t n, int dtype, double *d_work, void *stream);
int cszp2_compress_prepare_range(const void *d_in, uint64_t n, int dtype, double eb,
                                 const double *d_range, void *d_out, void *stream);

/* cszp2_compress_encode with ablation flags (NEXT #2; same stream bytes either way):
 *  CSZP2_FLAG_CHAINED_SCAN: replace the decoupled lookback by the plain chained
 *    scan it improves on (Fig 12 left; the Fig 17 comparison).
 *  CSZP2_FLAG_LOAD_VEC: each thread loads its own 32-value block with 16-byte
 *    vector loads (the paper's vectorised access, Fig 10-11) instead
 *    of the TMA tensor tiles.
 *  CSZP2_FLAG_LOAD_SCALAR: each thread loads its block value by value (the
 *    non-vectorised baseline of the §VI-E memory ablation).
 *  LOAD_VEC and LOAD_SCALAR are exclusive (ARG otherwise).
 *  CSZP2_FLAG_LB_WIDE / CSZP2_FLAG_LB_NARROW: force the lookback's first window
 *    to 256 / 32 predecessors (by default 32 below 2^16 tiles, 256 from 2^16 on; a speed
 *    choice that changes no stream byte). Exclusive (ARG otherwise). They apply to the
 *    TMA-load product path; the LOAD_* ablations keep 256, CHAINED_SCAN has no window.
 *  CSZP2_FLAG_PREPARED (not an ablation): the caller guarantees that a
 *    cszp2_compress_prepare(_range) on this d_out precedes this call on the stream
 *    with no encode in between, so the tile index and ticket are still zero and
 *    encode skips re-zeroing them (one launch less; cszp2_compress uses it). With
 *    the flag and no such prepare, the stream is undefined. */
#define CSZP2_FLAG_CHAINED_SCAN 1u
#define CSZP2_FLAG_LOAD_VEC 2u
#define CSZP2_FLAG_LOAD_SCALAR 4u
#define CSZP2_FLAG_PREPARED 8u
#define CSZP2_FLAG_LB_WIDE 16u
#define CSZP2_FLAG_LB_NARROW 32u
int cszp2_compress_encode_ex(const void *d_in, uint64_t n, int dtype, double eb, int eb_mode,
                             int enc_mode, void *d_out, uint64_t *d_out_bytes, unsigned flags,
                             void *stream);

/* Decompression (❸ locate → ❹ → ❷ → ❶ in one kernel).
 *  d_cmp    : a stream produced by cszp2_compress for the same (n, dtype),
 *             device, 16-byte aligned.
 *  d_out    : n values of `dtype`, device, 16-byte aligned.
 *  d_status : nullable DEVICE int. If non-null it is OR-ed with a nonzero
 *             code (CSZP2_ERR_FORMAT / CSZP2_ERR_RANGE) when the stream is
 *             invalid or has RANGE status (d_out is then unspecified). The
 *             caller zeroes it beforehand. */
int cszp2_decompress(const void *d_cmp, void *d_out, uint64_t n, int dtype, int *d_status,
                     void *stream);

/* Ablation (NEXT #2): a one-CTA-per-tile decompression kernel in two variants
 * that differ only in how a tile's payload start is found:
 *  CSZP2_LOCATE_LOOKBACK: the paper's way (❸ runs again in decompression)
 *    — the tile's payload bytes recomputed from its offset bytes, then a
 *    decoupled lookback over a caller-provided scratch array;
 *  CSZP2_LOCATE_INDEX: read from the persisted tile index (R-14).
 * Same output as cszp2_decompress.
 *  d_scratch : cszp2_decompress_scratch_bytes(n) bytes of device memory, zeroed
 *              by this call (asynchronously, on `stream`; used by LOOKBACK).
 *  other arguments as cszp2_decompress; ARG for an unknown `locate`. */
#define CSZP2_LOCATE_INDEX 0
#define CSZP2_LOCATE_LOOKBACK 1
uint64_t cszp2_decompress_scratch_bytes(uint64_t n);
int cszp2_decompress_tilewise(const void *d_cmp, void *d_out, uint64_t n, int dtype, int locate,
                              void *d_scratch, int *d_status, void *stream);

/* Random-access decompression (§VI-B): decode only the values
 * [first, first + count) of a stream of n values into d_out[0 .. count)
 * (device, any 4/8-byte alignment). Only the tiles (256 blocks = 8192 values)
 * covering the range are read; each is located in O(1) through the stream's
 * tile index (FORMAT.md §2). d_status as in cszp2_decompress. Errors: ARG if
 * the range exceeds n. */
int cszp2_decompress_range(const void *d_cmp, uint64_t n, int dtype, uint64_t first,
                           uint64_t count, void *d_out, int *d_status, void *stream);

/* Copy the 64-byte header of a device stream to the host and decode it.
 * Synchronises `stream`. */
int cszp2_read_header(const void *d_cmp, cszp2_header *h_hdr, void *stream);

/* End-to-end variants with HOST buffers (bench e2e). The caller provides
 * device work buffers (d_in_work: n*w bytes; d_out_work: compress bound);
 * host buffers should be pinned for full PCIe speed.
 * cszp2_compress_host: H2D copy of h_in, cszp2_compress, D2H copy of the
 *   stream into h_out (capacity h_out_cap); *h_out_bytes = stream bytes.
 *   Synchronises `stream`.
 * cszp2_decompress_host: H2D copy of h_cmp (cmp_bytes) into d_cmp_work,
 *   cszp2_decompress into d_out_work, D2H of n values into h_out.
 *   d_status as in cszp2_decompress (nullable); its value is returned if
 *   nonzero. Synchronises `stream`. */
int cszp2_compress_host(const void *h_in, uint64_t n, int dtype, double eb, int eb_mode,
                        int enc_mode, void *d_in_work, void *d_out_work, void *h_out,
                        uint64_t h_out_cap, uint64_t *h_out_bytes, void *stream);
int cszp2_decompress_host(const void *h_cmp, uint64_t cmp_bytes, void *d_cmp_work,
                          void *d_out_work, void *h_out, uint64_t n, int dtype, int *d_status,
                          void *stream);

/* Multi-GPU container index: exclusive prefix sum of the
 * per-rank stream sizes gathered from every rank's d_out_bytes.
 *  d_sizes   : nparts device uint64 (all-gathered sizes, rank order).
 *  d_offsets : nparts + 1 device uint64; d_offsets[r] = Σ_{j<r} d_sizes[j],
 *              d_offsets[nparts] = total container bytes. */
int cszp2_container_index(const uint64_t *d_sizes, int nparts, uint64_t *d_offsets,
                          void *stream);

/* ---- Multi-dimensional Lorenzo layouts (§VI-D,
 * Table VI; FORMAT.md §7). The paper's 2D (8x8 block) and 3D (4x4x4 block)
 * variants of the same single-kernel design: L = 64 values per block, residual =
 * value − Lorenzo prediction from the 3 (2D) / 7 (3D) lower in-block neighbours
 * (neighbours outside the block are 0), then the same Plain/Outlier FLE (8-byte
 * bit fields) and decoupled-lookback concatenation. The stream carries predictor
 * id and nx, ny in its header (a 1D decoder refuses it, and vice versa).
 *  field      : nx * ny (* nz) values of `dtype`, row-major with x fastest,
 *               device, 16-byte aligned. ndim = 2 requires nz = 1.
 *  extents    : nx, ny, nz < 2^32 and nx*ny*nz <= 2^35 (the 1D limit), else ARG,
 *               for compression and decompression alike.
 * cszp2_compress_bound_nd: bytes d_out must hold (0 on bad arguments), including
 *   16 bytes of scratch past the stream, as cszp2_compress_bound.
 * cszp2_compress_nd: like cszp2_compress (same eb / eb_mode / enc_mode meaning,
 *   same RANGE behaviour with this predictor's tighter limit |x/2eb| <= 2^28-1 (2D)
 *   or 2^27-1 (3D), FORMAT.md §7); asynchronous on `stream`.
 * cszp2_compress_nd_ex: the same with flags: CSZP2_FLAG_LB_WIDE / CSZP2_FLAG_LB_NARROW
 *   as for cszp2_compress_encode_ex (same stream bytes either way); any other bit, or
 *   both, is ARG.
 * cszp2_decompress_nd: inverse; d_out = nx*ny*nz values, device, 16-byte aligned;
 *   d_status as in cszp2_decompress. */
uint64_t cszp2_compress_bound_nd(uint64_t nx, uint64_t ny, uint64_t nz, int ndim, int dtype);
int cszp2_compress_nd(const void *d_in, uint64_t nx, uint64_t ny, uint64_t nz, int ndim, int dtype,
                      double eb, int eb_mode, int enc_mode, void *d_out, uint64_t *d_out_bytes,
                      void *stream);
int cszp2_compress_nd_ex(const void *d_in, uint64_t nx, uint64_t ny, uint64_t nz, int ndim, int dtype,
                         double eb, int eb_mode, int enc_mode, void *d_out, uint64_t *d_out_bytes,
                         unsigned flags, void *stream);
int cszp2_decompress_nd(const void *d_cmp, void *d_out, uint64_t nx, uint64_t ny, uint64_t nz, int ndim,
                        int dtype, int *d_status, void *stream);

/* Library identification ("cszp2 <version> sm_100a"). */
const char *cszp2_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CSZP2_H */
