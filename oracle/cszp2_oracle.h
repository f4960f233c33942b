/*
 * cszp2_oracle.h — plain, slow, single-threaded CPU oracle for the cuSZp2
 * compressor (Huang et al., SC'24; PAPER.md). TEST INFRASTRUCTURE ONLY:
 * only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it. The product path never does.
 *
 * It follows FORMAT.md step by step in the paper's order
 *   ❶ lossy conversion → first-order difference
 *   → ❷ Plain/Outlier FLE → ❸ serial prefix sum
 *   → ❹ concatenation
 * and shares no code, header, table or constant with the CUDA path.
 *
 * Parity pins: see tests/test_oracle_pins.py and DESIGN.md §4.
 * Pinned: quantization (paper example P:122, eb = 0.5 textbook rint, error
 * bound), sizes, Outlier ≤ Plain, same
 * reconstruction P vs O, serial prefix, bit layout (an
 * independent numpy bit parser), REL range (numpy min/max).
 * Parity unpinned: none of the functions below.
 */
#ifndef CSZP2_ORACLE_H
#define CSZP2_ORACLE_H
#include <stdint.h>

#define ORC_F32 0
#define ORC_F64 1
#define ORC_ABS 0
#define ORC_REL 1
#define ORC_PLAIN 0
#define ORC_OUTLIER 1
#define ORC_OK 0
#define ORC_ERR_ARG 1
#define ORC_ERR_RANGE 3
#define ORC_ERR_FORMAT 4

/* FORMAT.md §2: bytes a stream of n values may need. */
uint64_t oracle_compress_bound(uint64_t n, int L);

/* FORMAT.md §6.1: ABS -> eb; REL -> lambda * (max - min). */
int oracle_resolve_eb(const void *x, uint64_t n, int dtype, double eb, int eb_mode,
                      double *eb_abs);

/* FORMAT.md §6.3: q[i] = rint(x[i] * inv). Returns ORC_OK or ORC_ERR_RANGE. */
int oracle_quantize(const void *x, uint64_t n, int dtype, double eb_abs, int32_t *q);

/* FORMAT.md §6.6: x'[i] = (T)q[i] * s. */
void oracle_dequantize(const int32_t *q, uint64_t n, int dtype, double eb_abs, void *x);

/* FORMAT.md §6.4-6.5: one block of L quantization integers (tail
 * already padded) -> offset byte + payload. Returns the payload size. */
int oracle_encode_block(const int32_t *q, int L, int enc_mode, uint8_t *offset_byte,
                        uint8_t *payload);

/* Inverse of oracle_encode_block. Returns the payload size consumed, or -1 for
 * an invalid offset byte. */
int oracle_decode_block(uint8_t offset_byte, const uint8_t *payload, int L, int32_t *q);

/* Payload size implied by an offset byte alone (-1 if invalid). */
int oracle_block_size(uint8_t offset_byte, int L);

/* Whole stream. out must hold oracle_compress_bound(n, L) bytes. Returns
 * ORC_OK, ORC_ERR_ARG or ORC_ERR_RANGE (a RANGE stream is still written:
 * header with status 3). */
int oracle_compress(const void *x, uint64_t n, int dtype, double eb, int eb_mode,
                    int enc_mode, int L, uint8_t *out, uint64_t *out_bytes);

/* Lossless part only: n given quantization integers -> stream (dtype field 0,
 * eb fields 0). Used by the brute-force encoder tests. */
int oracle_compress_ints(const int32_t *q, uint64_t n, int enc_mode, int L, uint8_t *out,
                         uint64_t *out_bytes);

/* Whole-stream inverse. Returns ORC_OK, ORC_ERR_RANGE or ORC_ERR_FORMAT. */
int oracle_decompress(const uint8_t *cmp, uint64_t cmp_bytes, void *out, uint64_t n,
                      int dtype);

/* Lossless inverse of oracle_compress_ints. */
int oracle_decompress_ints(const uint8_t *cmp, uint64_t cmp_bytes, int32_t *q, uint64_t n);

/* NEXT #3 (Table VI; FORMAT.md §7): 2D Lorenzo on 8x8 blocks / 3D Lorenzo on
 * 4x4x4 blocks of an nx x ny (x nz) field (x fastest), L = 64, same FLE. */
uint64_t oracle_compress_bound_nd(uint64_t nx, uint64_t ny, uint64_t nz, int ndim);
int oracle_compress_nd(const void *x, uint64_t nx, uint64_t ny, uint64_t nz, int ndim,
                       int dtype, double eb, int eb_mode, int enc_mode, uint8_t *out,
                       uint64_t *out_bytes);
int oracle_decompress_nd(const uint8_t *cmp, uint64_t cmp_bytes, void *out, uint64_t nx,
                         uint64_t ny, uint64_t nz, int ndim, int dtype);

#endif
