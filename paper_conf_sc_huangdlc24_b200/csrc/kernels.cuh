// kernels.cuh — sm_100a kernels of the cuSZp2 hot path (FORMAT.md; PAPER.md).
//
//   minmax_kernel      REL -> ABS: grid-wide exact min/max, eb_abs = λ·(max−min)
//   compress_kernel    ❶ pre-quantization → in-block 1D Lorenzo → ❷ Plain/Outlier
//                      FLE → ❸ decoupled-lookback exclusive scan → ❹ concatenation,
//                      one fused pass (Fig 4)
//   decompress_kernel  ❸ (O(1) from the persisted tile index) → ❹ → ❷⁻¹ → ❶⁻¹
//
// B200 design: persistent CTAs that claim tiles of 256 blocks (8192 f32
// values) in order from an atomic ticket (compression) or walk tiles c, c+G, ...
// (decompression); one thread = one 32-value block (block-level data parallelism,
// P:176). Tiles move between HBM and shared memory with TMA: 2D tensor maps with
// 128-byte swizzle for the dense value side (so thread-per-block 16-byte shared
// accesses are bank-conflict free), 1D bulk copies for the byte-granular compressed
// side. Bit planes are packed/unpacked by in-register 32x32 bit transposes sized to
// the warp's largest fixed length.
#pragma once
#include <cstdint>
#include <type_traits>
#include <cuda.h>

#include "ptx.cuh"

namespace cszp2 {

#ifdef CSZP2_TRACE
// debug build only: per-tile globaltimer stamps [claim, data, publishA, resolved, written, polls]
__device__ uint64_t *g_trace = nullptr;
__device__ __forceinline__ uint64_t gtimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#define TRACE(tile, slot, val) \
    do { if (g_trace) g_trace[(tile) * 16 + (slot)] = (val); } while (0)
#else
#define TRACE(tile, slot, val) do { } while (0)
#endif

#ifdef CSZP2_WD
// debug build only (hang hunting): spinning sites report their state into host-mapped
// memory, 8 records of 8 words per CTA, read by the host while the kernel runs
__device__ uint64_t *g_wd = nullptr;
#define WD_REC(site, a, b, c, d)                                                          \
    do {                                                                                  \
        if (g_wd) {                                                                       \
            volatile uint64_t *r_ = g_wd + (static_cast<uint64_t>(blockIdx.x) * 8 + (site)) * 8; \
            r_[1] = (a);                                                                  \
            r_[2] = (b);                                                                  \
            r_[3] = (c);                                                                  \
            r_[4] = (d);                                                                  \
            r_[0] = (site) | (static_cast<uint64_t>(threadIdx.x) << 8) | (1ull << 40);    \
        }                                                                                 \
    } while (0)
#else
#define WD_REC(site, a, b, c, d) do { } while (0)
#endif

constexpr int L = 32;      // values per block
constexpr int BPT = 256;   // blocks per tile (FORMAT.md §1)
constexpr int NT = 256;    // threads per CTA: one block per thread
constexpr int TMA_TID = 32;  // compression: the thread that claims tiles and owns the TMA traffic
constexpr uint32_t MAGIC = 0x325A5343u;
constexpr uint64_t FLAG_A = 1ull << 62;   // lookback: aggregate available
constexpr uint64_t FLAG_P = 2ull << 62;   // lookback: inclusive prefix available
constexpr uint64_t VAL_MASK = (1ull << 62) - 1;
constexpr int ST_RANGE = 3;
constexpr int ST_FORMAT = 4;

struct Geom {
    uint64_t n;      // values
    uint64_t nb;     // blocks = ceil(n / L)
    uint64_t nfull;  // blocks with all L values = n / L
    uint64_t T;      // tiles
    uint64_t O;      // offset-byte region start
    uint64_t D;      // payload region start
};

__host__ __device__ inline uint64_t roundup16(uint64_t v) { return (v + 15) & ~uint64_t(15); }

template <typename T>
struct Traits;
template <>
struct Traits<float> {
    static constexpr int ROWS = 1;  // 128-byte TMA rows per block
    static constexpr int TILE_BYTES = BPT * L * 4;
    static constexpr int DTYPE = 0;
};
template <>
struct Traits<double> {
    static constexpr int ROWS = 2;
    static constexpr int TILE_BYTES = BPT * L * 8;
    static constexpr int DTYPE = 1;
};

// ------------------------------------------------------------------ arithmetic contract
// FORMAT.md §6.2-6.3 / §6.6: RN multiply (no FMA), round-half-even conversion.
struct ConstsF {
    float inv, s;
    bool ok;
};
struct ConstsD {
    double inv, s;
    bool ok;
};
__device__ __forceinline__ ConstsF make_consts(double eb, float *) {
    ConstsF c;
    c.inv = __double2float_rn(__ddiv_rn(1.0, __dmul_rn(2.0, eb)));
    c.s = __double2float_rn(__dmul_rn(2.0, eb));
    c.ok = (eb > 0.0) && isfinite(eb) && (c.inv > 0.0f) && isfinite(c.inv) && (c.s > 0.0f) &&
           isfinite(c.s);
    return c;
}
__device__ __forceinline__ ConstsD make_consts(double eb, double *) {
    ConstsD c;
    c.inv = __ddiv_rn(1.0, __dmul_rn(2.0, eb));
    c.s = __dmul_rn(2.0, eb);
    c.ok = (eb > 0.0) && isfinite(eb) && (c.inv > 0.0) && isfinite(c.inv) && (c.s > 0.0) &&
           isfinite(c.s);
    return c;
}
__device__ __forceinline__ int quantize(float x, float inv, bool &bad) {
    float t = __fmul_rn(x, inv);
    bad |= !(fabsf(t) <= 1073741760.0f);  // also true for NaN
    return __float2int_rn(t);
}
__device__ __forceinline__ int quantize(double x, double inv, bool &bad) {
    double t = __dmul_rn(x, inv);
    bad |= !(fabs(t) <= 1073741823.0);
    return __double2int_rn(t);
}
// Whole-block ❶ for the 1D compressor, bit-identical to quantize() above but without the
// slow F2I conversions (1/8-rate pipe) in the common case: for |t| < 2^22,
// fl(t + 1.5·2^23) lies in [2^23, 2^24) where the float spacing is 1, so the RN addition
// rounds t half-to-even to an integer that is read straight out of the bit pattern.
// A block with any |t| >= 2^22 (or NaN) takes the F2I path with the full range check.
// Output is BIASED: qb_i = q_i + QBIAS (mod 2^32), so that the bit patterns can be
// differenced directly (d_i = qb_i - qb_{i-1}, q_{-1} = 0 <=> qb_{-1} = QBIAS).
// (f64: fl(t + 1.5·2^52) does the same for every |t| < 2^51; its low word is rint(t).)
template <typename T>
struct QBias;
template <>
struct QBias<float> {
    static constexpr int value = 0x4B400000;
};
template <>
struct QBias<double> {
    static constexpr int value = 0;
};
__device__ __forceinline__ void quantize_block(const float (&x)[L], float inv, int (&qb)[L], bool &bad) {
    bool big[4] = {false, false, false, false};  // independent predicate chains
#pragma unroll
    for (int i = 0; i < L; i++) {
        const float t = __fmul_rn(x[i], inv);
        qb[i] = __float_as_int(__fadd_rn(t, 12582912.0f));
        big[i & 3] |= !(fabsf(t) < 4194304.0f);
    }
    if ((big[0] || big[1]) || (big[2] || big[3])) {
#pragma unroll
        for (int i = 0; i < L; i++) {
            const float t = __fmul_rn(x[i], inv);
            bad |= !(fabsf(t) <= 1073741760.0f);
            qb[i] = static_cast<int>(static_cast<uint32_t>(__float2int_rn(t)) + 0x4B400000u);
        }
    }
}
// The same biased patterns with no range check at all. They are exact whenever the
// block's differences (taken from these patterns, q_{-1} = QBIAS) all satisfy
// |d_i| < 2^17: then every |qb_i - QBIAS| <= 32 (2^17 - 1) < 2^22, so each
// s_i = fl(t_i + 1.5·2^23) has its bit pattern strictly inside (2^23, 2^24) — which
// rounding can only produce from t_i + 1.5·2^23 in [2^23, 2^24), where the RN addition
// is rint(t_i) exactly and |t_i| < 2^22 passes the range check (NaN and ±Inf have
// patterns outside that interval). The caller redoes a block with fl_p > 17 through
// quantize_block().
constexpr int FAST_FL_MAX = 17;
__device__ __forceinline__ void quantize_block_unchecked(const float (&x)[L], float inv, int (&qb)[L]) {
#pragma unroll
    for (int i = 0; i < L; i++) qb[i] = __float_as_int(__fadd_rn(__fmul_rn(x[i], inv), 12582912.0f));
}
__device__ __forceinline__ void quantize_block(const double (&x)[L], double inv, int (&qb)[L], bool &bad) {
#pragma unroll
    for (int i = 0; i < L; i++) {
        const double t = __dmul_rn(x[i], inv);
        bad |= !(fabs(t) <= 1073741823.0);
        qb[i] = static_cast<int>(static_cast<uint32_t>(__double_as_longlong(__dadd_rn(t, 6755399441055744.0))));
    }
}
__device__ __forceinline__ float dequantize(int q, float s) { return __fmul_rn(__int2float_rn(q), s); }
__device__ __forceinline__ double dequantize(int q, double s) {
    return __dmul_rn(__int2double_rn(q), s);
}

// Align a dynamic shared-memory pointer by offsetting the __shared__ array itself (an
// integer round trip through uintptr_t would lose the address space, and every access
// through the result would compile to a generic LD.E/ST.E with 64-bit address math).
template <uint32_t A>
__device__ __forceinline__ uint8_t *smem_align(uint8_t *raw) {
    return raw + ((A - (smem_u32(raw) & (A - 1))) & (A - 1));
}

// ------------------------------------------------------------------ swizzled tile access
// TMA SWIZZLE_128B: the 16-byte chunk c of 128-byte row r lives at chunk c ^ (r & 7).
__device__ __forceinline__ uint32_t swz(uint32_t row, uint32_t chunk) {
    return row * 128u + ((chunk ^ (row & 7u)) << 4);
}
__device__ __forceinline__ void load_block(const uint8_t *tile, uint32_t r, float (&x)[L]) {
    // row base | (r & 7) << 4 is loop-invariant; chunk c is then one XOR away
    const uint32_t base = smem_u32(tile) + r * 128u + ((r & 7u) << 4);
#pragma unroll
    for (int c = 0; c < 8; c++) {
        float4 v;
        asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                     : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                     : "r"(base ^ (static_cast<uint32_t>(c) << 4)));
        x[4 * c + 0] = v.x;
        x[4 * c + 1] = v.y;
        x[4 * c + 2] = v.z;
        x[4 * c + 3] = v.w;
    }
}
__device__ __forceinline__ void load_block(const uint8_t *tile, uint32_t r, double (&x)[L]) {
#pragma unroll
    for (int h = 0; h < 2; h++)
#pragma unroll
        for (int c = 0; c < 8; c++) {
            double2 v = *reinterpret_cast<const double2 *>(tile + swz(2 * r + h, c));
            x[16 * h + 2 * c + 0] = v.x;
            x[16 * h + 2 * c + 1] = v.y;
        }
}
__device__ __forceinline__ void store_block(uint8_t *tile, uint32_t r, const float (&x)[L]) {
#pragma unroll
    for (int c = 0; c < 8; c++)
        *reinterpret_cast<float4 *>(tile + swz(r, c)) =
            make_float4(x[4 * c], x[4 * c + 1], x[4 * c + 2], x[4 * c + 3]);
}
__device__ __forceinline__ void store_block(uint8_t *tile, uint32_t r, const double (&x)[L]) {
#pragma unroll
    for (int h = 0; h < 2; h++)
#pragma unroll
        for (int c = 0; c < 8; c++)
            *reinterpret_cast<double2 *>(tile + swz(2 * r + h, c)) =
                make_double2(x[16 * h + 2 * c], x[16 * h + 2 * c + 1]);
}

// ------------------------------------------------------------------ byte-granular smem access
__device__ __forceinline__ uint32_t ld_u32_unaligned(const uint8_t *base, uint32_t pos) {
    const uint32_t *w = reinterpret_cast<const uint32_t *>(base + (pos & ~3u));
    return __funnelshift_r(w[0], w[1], 8u * (pos & 3u));
}

// ------------------------------------------------------------------ bit-plane transposes
// A 32x32 bit matrix in 32 registers (row r = A[r], column c = bit c) transposes
// in five stages; stage s exchanges the s-bit off-diagonal blocks of every 2s x 2s
// block (it swaps bit log2(s) of the row index with that of the column index, so the
// stages commute). When only the first R = 2^M columns can be nonzero, the stages
// s >= R reduce to merges A[i] |= A[i+s] << s (rows [s, 2s) become zero) and the
// remaining ones touch rows [0, R) only. Cost per 32 values: R=1: 31 ops, 2: 35,
// 4: 48, 8: 84, 16: 176, 32: 400 — against 64 per plane for a bit-serial pack.
// (Byte permutes (PRMT) for the S = 16 / 8 stages measured -1% on both kernels.)
__host__ __device__ constexpr uint32_t stage_mask(int s) {
    return s == 16 ? 0x0000FFFFu
                   : (s == 8 ? 0x00FF00FFu : (s == 4 ? 0x0F0F0F0Fu : (s == 2 ? 0x33333333u : 0x55555555u)));
}
template <int S, int ROWS>
__device__ __forceinline__ void swap_stage(uint32_t (&A)[32]) {
#pragma unroll
    for (int i = 0; i < ROWS; i++) {
        if ((i & S) == 0) {
            const uint32_t t = ((A[i] >> S) ^ A[i + S]) & stage_mask(S);
            A[i + S] ^= t;
            A[i] ^= t << S;
        }
    }
}
// values (bits < 2^M) -> planes: A[k] = sum_i bit_k(value_i) << i, k < 2^M
template <int S>
__device__ __forceinline__ void merge_stage(uint32_t (&A)[32]) {
#pragma unroll
    // the bits are disjoint, so + is |: one IMAD or LEA per row instead of SHL + LOP3
    for (int i = 0; i < S; i++) A[i] = A[i + S] * (1u << S) + A[i];
}
template <int S>
__device__ __forceinline__ void split_stage(uint32_t (&A)[32]) {
#pragma unroll
    for (int i = 0; i < S; i++) {
        A[i + S] = (A[i] >> S) & stage_mask(S);
        A[i] &= stage_mask(S);
    }
}
template <int M>
__device__ __forceinline__ void pack_planes(uint32_t (&A)[32]) {
    constexpr int R = 1 << M;
    if constexpr (R <= 16) merge_stage<16>(A);
    if constexpr (R <= 8) merge_stage<8>(A);
    if constexpr (R <= 4) merge_stage<4>(A);
    if constexpr (R <= 2) merge_stage<2>(A);
    if constexpr (R <= 1) merge_stage<1>(A);
    if constexpr (M >= 5) swap_stage<16, R>(A);
    if constexpr (M >= 4) swap_stage<8, R>(A);
    if constexpr (M >= 3) swap_stage<4, R>(A);
    if constexpr (M >= 2) swap_stage<2, R>(A);
    if constexpr (M >= 1) swap_stage<1, R>(A);
}
// planes (rows >= fl zero, rows >= 2^M don't care) -> values: A[i] = sum_k bit_i(plane_k) << k
template <int M>
__device__ __forceinline__ void unpack_planes(uint32_t (&A)[32]) {
    constexpr int R = 1 << M;
    if constexpr (M >= 1) swap_stage<1, R>(A);
    if constexpr (M >= 2) swap_stage<2, R>(A);
    if constexpr (M >= 3) swap_stage<4, R>(A);
    if constexpr (M >= 4) swap_stage<8, R>(A);
    if constexpr (M >= 5) swap_stage<16, R>(A);
    if constexpr (R <= 1) split_stage<1>(A);
    if constexpr (R <= 2) split_stage<2>(A);
    if constexpr (R <= 4) split_stage<4>(A);
    if constexpr (R <= 8) split_stage<8>(A);
    if constexpr (R <= 16) split_stage<16>(A);
}
// p ? a : b through selp, which the front end cannot turn into an indexed load
__device__ __forceinline__ uint32_t opaque_select(bool p, uint32_t a, uint32_t b) {
    uint32_t r;
    asm("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %1, 0;\n\tselp.b32 %0, %2, %3, q;\n\t}"
        : "=r"(r)
        : "r"(static_cast<uint32_t>(p)), "r"(a), "r"(b));
    return r;
}
// smallest M with fl <= 2^M (fl in 1..31)
__device__ __forceinline__ int plane_log2(int fl) { return fl <= 1 ? 0 : 32 - __clz(fl - 1); }

// One block's payload to smem at byte address `st` (any alignment): sign word, nob
// outlier bytes, then planes A[0..fl). Let ps = st + 4 + nob (plane region), r = ps & 3
// and P_k the 4 payload bytes at ps + 4k (P_-1, P_-2: header bytes before ps). Every
// aligned word at ps - r + 4k is funnel(P_k-1, P_k, 8r); those wholly inside the block
// (k = 0..fl-1, and k = -1 when nob >= r) are plain 32-bit stores. The <= 4 head and
// <= 3 tail bytes share an aligned word with a neighbouring block: the staging area is
// kept zeroed outside live payloads (the resolver clears what it has copied out), so
// each of the two partial words is merged with a single shared-memory atomicOr.
// SIMT-uniform: no data-dependent branches.
template <int R>
__device__ __forceinline__ void stage_payload(uint8_t *base, uint32_t st, uint32_t sign,
                                              uint32_t outl, int nob, int fl,
                                              const uint32_t (&A)[32]) {
    const uint64_t hdr = sign | (static_cast<uint64_t>(outl) << 32);
    const uint32_t ps = st + 4u + nob;
    const uint32_t r = ps & 3u;
    const uint32_t sh = 8u * r;
    const uint32_t pm1 = static_cast<uint32_t>(hdr >> (8 * nob));                // P_-1
    const uint32_t pm2 = static_cast<uint32_t>(hdr << (32 - 8 * nob));           // P_-2 (top nob bytes)
    uint32_t *w = reinterpret_cast<uint32_t *>(base + ps - r);                   // word k at w[k]
    const bool wm1 = static_cast<uint32_t>(nob) >= r;
    if (wm1) w[-1] = __funnelshift_l(pm2, pm1, sh);
    const uint32_t hw = ps - r - (wm1 ? 4u : 0u);  // aligned end of the head bytes
    const uint32_t head = hw - st;                 // 0..4 bytes: the top bytes of word hw - 4
    if (head) atomicOr(reinterpret_cast<unsigned *>(base + hw - 4), static_cast<uint32_t>(hdr) << (32 - 8 * head));
    uint32_t prev = pm1, top = pm1;
#pragma unroll
    for (int k = 0; k < R; k++) {
        if (k < fl) {
            w[k] = __funnelshift_l(prev, A[k], sh);
            prev = A[k];
        }
        top = opaque_select(k < fl, A[k], top);
    }
    const uint32_t e = ps + 4u * fl;  // end of the payload; its last r bytes are the low bytes of word e - r
    if (r) atomicOr(reinterpret_cast<unsigned *>(base + e - r), top >> (32 - sh));
}

// Planes 0..fl-1 of one block from smem at byte position `pos` (any alignment) into
// A[0..R): rows >= fl are zeroed; each plane is a funnel of two aligned words.
template <int R>
__device__ __forceinline__ void load_planes(const uint8_t *base, uint32_t pos, uint32_t fl,
                                            uint32_t (&A)[32]) {
    const uint32_t *w = reinterpret_cast<const uint32_t *>(base + (pos & ~3u));
    const uint32_t sh = 8u * (pos & 3u);
    uint32_t lo = w[0];
#pragma unroll
    for (int k = 0; k < R; k++) {
        uint32_t v = 0;
        if (k < (int)fl) {
            const uint32_t hi = w[k + 1];
            v = __funnelshift_r(lo, hi, sh);
            lo = hi;
        }
        A[k] = v;
    }
}

// ------------------------------------------------------------------ scans
// Exclusive scan of one u32 per thread over the NT threads 0..NT-1, synchronised
// with barrier `bar_id` (0 = the whole CTA). Returns the exclusive prefix;
// *total receives the sum. Contains two barriers.
__device__ __forceinline__ void group_sync(uint32_t bar_id) {
    if (bar_id == 0)
        __syncthreads();
    else
        named_sync(bar_id, NT);
}
__device__ __forceinline__ uint32_t cta_exclusive_scan(uint32_t v, uint32_t *s_warp,
                                                       uint32_t *total, uint32_t bar_id = 0) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) s_warp[warp] = inc;
    group_sync(bar_id);
    // every warp scans the NT/32 warp totals itself (3 shuffle steps)
    constexpr int NW = NT / 32;
    uint32_t wt = lane < NW ? s_warp[lane] : 0u;
#pragma unroll
    for (int o = 1; o < NW; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, wt, o);
        if (lane >= o) wt += y;
    }
    const uint32_t before = __shfl_sync(0xffffffffu, wt, (warp + NW - 1) % NW);
    *total = __shfl_sync(0xffffffffu, wt, NW - 1);
    group_sync(bar_id);
    return (warp ? before : 0u) + inc - v;
}

// The compressor's intra-tile scan with ONE barrier: the warp totals (bit 31: some
// block of the warp was flagged `bad`; a warp's payload total is < 2^31) go to
// s_warp, which the caller double-buffers by tile parity — a warp can only rewrite
// a buffer after the next tile's barrier, which every warp reaches only after reading
// this tile's totals. Also returns the OR of `bad` over the tile.
__device__ __forceinline__ uint32_t tile_scan_1bar(uint32_t v, bool bad, uint32_t *s_warp,
                                                   uint32_t *total, bool *any_bad, uint32_t bar_id) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    const bool wbad = __any_sync(0xffffffffu, bad);
    if (lane == 31) s_warp[warp] = inc | (wbad ? 0x80000000u : 0u);
    named_sync(bar_id, NT);
    constexpr int NW = NT / 32;
    const uint32_t raw = lane < NW ? s_warp[lane] : 0u;
    *any_bad = __any_sync(0xffffffffu, (raw >> 31) != 0u);
    uint32_t wt = raw & 0x7FFFFFFFu;
#pragma unroll
    for (int o = 1; o < NW; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, wt, o);
        if (lane >= o) wt += y;
    }
    const uint32_t before = __shfl_sync(0xffffffffu, wt, (warp + NW - 1) % NW);
    *total = __shfl_sync(0xffffffffu, wt, NW - 1);
    return (warp ? before : 0u) + inc - v;
}

// tile_scan_1bar split around a barrier the caller already has: part 1 (warp scan, warp
// total + bad flag to s_warp) before it, part 2 (warp totals -> exclusive prefix, tile
// total, OR of bad) after it.
__device__ __forceinline__ uint32_t scan_part1(uint32_t v, bool bad, uint32_t *s_warp) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    const bool wbad = __any_sync(0xffffffffu, bad);
    if (lane == 31) s_warp[warp] = inc | (wbad ? 0x80000000u : 0u);
    return inc;
}
__device__ __forceinline__ uint32_t scan_part2(uint32_t v, uint32_t inc, const uint32_t *s_warp, uint32_t *total,
                                               bool *any_bad) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    constexpr int NW = NT / 32;
    const uint32_t raw = lane < NW ? s_warp[lane] : 0u;
    *any_bad = __any_sync(0xffffffffu, (raw >> 31) != 0u);
    uint32_t wt = raw & 0x7FFFFFFFu;
#pragma unroll
    for (int o = 1; o < NW; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, wt, o);
        if (lane >= o) wt += y;
    }
    const uint32_t before = __shfl_sync(0xffffffffu, wt, (warp + NW - 1) % NW);
    *total = __shfl_sync(0xffffffffu, wt, NW - 1);
    return (warp ? before : 0u) + inc - v;
}

// ❸ Decoupled lookback (Fig 13; after Merrill & Garland [25]), split
// so that no CTA ever sits on an unpublished tile while it waits:
//   publish_aggregate: tile t announces (A | aggregate) — (P | aggregate) for
//                      tile 0 — as soon as its blocks are encoded;
//   lookback_issue /   one iteration later, a full warp loads its predecessors'
//   lookback_finish:   descriptors in windows of 256 (8 per lane, nearest first;
//                      loads issued before the next tile's encode so their latency
//                      hides behind it), sums aggregates down to the nearest
//                      inclusive prefix (P) and publishes (P | inclusive).
// Descriptor: flag (bits 63-62: 0 Waiting, 1 A, 2 P) | RANGE bit 61 (A: this
// tile saw an out-of-range value; P: some tile <= t did) | value (bits 60-0).
// Nothing but the descriptors themselves is communicated through them, so all
// accesses are relaxed (no membar on the critical path). The final descriptors
// ARE the stream's tile index (FORMAT.md §2; bit 61 is 0 in every valid stream).
constexpr int LB_PER_LANE = 8;
constexpr uint64_t BIT_RANGE = 1ull << 61;
constexpr uint64_t VAL61 = BIT_RANGE - 1;

__device__ __forceinline__ void publish_aggregate(uint64_t *index, uint64_t t, uint64_t agg,
                                                  bool bad) {
    st_relaxed_u64(&index[t], (t == 0 ? FLAG_P : FLAG_A) | (bad ? BIT_RANGE : 0) | agg);
}

template <int ROWS = LB_PER_LANE>
struct LookbackWindow {
    uint64_t d[ROWS];
};

// Window rows: row u, lane l holds the descriptor of tile j − (32u + l) (nearest first;
// each row is one coalesced 256-byte load).
template <int ROWS>
__device__ __forceinline__ void lookback_issue(const uint64_t *index, int64_t j, LookbackWindow<ROWS> &w) {
    const int64_t base = j - (threadIdx.x & 31);
#pragma unroll
    for (int u = 0; u < ROWS; u++)
        w.d[u] = (base - 32 * u >= 0) ? ld_relaxed_u64(&index[base - 32 * u]) : FLAG_P;  // virtual P|0
}

// Returns the exclusive prefix of tile t (>= 1) and publishes its inclusive
// descriptor; *range_out = RANGE bit of the inclusive prefix. Slot (row u, lane l) has
// the nearest-first key 32u + l. Per window, a constant number of warp collectives
// (not one set per row): the nearest P and the nearest Waiting slot by two min
// reductions; if a Waiting slot is nearer than the P, the Waiting slots are re-polled;
// otherwise every slot before the P is an A, whose values (tile aggregates, each
// <= 256 * 132 bytes, so 256 of them fit in 32 bits) are summed by one reduction.
template <int ROWS>
__device__ __forceinline__ uint64_t lookback_finish(uint64_t *index, uint64_t t, uint64_t agg,
                                                    bool bad, LookbackWindow<ROWS> &w, bool *range_out) {
    const int lane = threadIdx.x & 31;
    uint64_t excl = 0;
    bool rb = bad;
    int64_t j = static_cast<int64_t>(t) - 1;  // nearest predecessor of the window
    while (true) {
        uint32_t pk = 0xFFFFu, wk = 0xFFFFu;
#pragma unroll
        for (int u = ROWS - 1; u >= 0; u--) {  // descending: the nearest row wins
            const uint32_t f = static_cast<uint32_t>(w.d[u] >> 62);
            if (f == 2) pk = 32u * u + lane;
            if (f == 0) wk = 32u * u + lane;
        }
        const uint32_t P = __reduce_min_sync(0xffffffffu, pk);
        const uint32_t W = __reduce_min_sync(0xffffffffu, wk);
        if (W < P) {  // a needed predecessor is still Waiting: re-poll the Waiting slots
#ifdef CSZP2_WD
            {
                static_assert(true, "");
                const uint64_t wd_t = t;
                if (lane == 0) WD_REC(6, wd_t, static_cast<uint64_t>(j), P, (static_cast<uint64_t>(W) << 32) | (t - 1 - j + W));
            }
#endif
#ifdef CSZP2_TRACE
            if (lane == 0 && g_trace) g_trace[t * 16 + 5]++;
#endif
            __nanosleep(32);
#pragma unroll
            for (int u = 0; u < ROWS; u++) {
                const int64_t idx = j - 32 * u - lane;
                if ((w.d[u] >> 62) == 0 && idx >= 0) w.d[u] = ld_relaxed_u64(&index[idx]);
            }
            continue;
        }
        uint32_t s = 0;
        bool r = false;
        uint64_t pv = 0;
#pragma unroll
        for (int u = 0; u < ROWS; u++) {
            const uint32_t key = 32u * u + lane;
            const uint64_t d = w.d[u];
            if (key < P) s += static_cast<uint32_t>(d);  // an A: value < 2^32
            if (key <= P) r |= (d & BIT_RANGE) != 0;
            if (key == P) pv = d & VAL61;
        }
        excl += __reduce_add_sync(0xffffffffu, s);
        rb |= __any_sync(0xffffffffu, r);
        if (P < 32u * ROWS) {
            excl += __shfl_sync(0xffffffffu, pv, P & 31u);
            break;
        }
#ifdef CSZP2_TRACE
        if (lane == 0 && g_trace) g_trace[t * 16 + 5] += 1ll << 32;  // extra window
#endif
        j -= 32 * ROWS;
        lookback_issue(index, j, w);
    }
    if (lane == 0) st_relaxed_u64(&index[t], FLAG_P | (rb ? BIT_RANGE : 0) | (excl + agg));
    *range_out = rb;
    return excl;
}

// Issue the first window and resolve (used by the compression consumer warp). Window
// width 32 x ROWS: the compressors are instantiated with 256 (ROWS = 8) and with 32
// (ROWS = 1, windows walked one row at a time); the launch takes 32 for fields of at
// most LB_NARROW_TILES tiles. Measured, not derived: on configs 2-4b (≤ 34k tiles) the
// 32-wide window is 3-10% faster (1D configs 3a/4a, the 3D kernel); on config 5's data it
// ties at 2^15 tiles and loses from 2^16 tiles on (4-8% at 2^17, a config 5 slab at 8 GPUs;
// 8-10% at 2^20) (profiles/ab_lookback_window_r02b.txt).
constexpr uint64_t LB_NARROW_TILES = (1ull << 16) - 1;
template <int ROWS = LB_PER_LANE>
__device__ __forceinline__ uint64_t lookback(uint64_t *index, uint64_t t, uint64_t agg, bool bad,
                                             bool *range_out) {
    LookbackWindow<ROWS> w;
    lookback_issue<ROWS>(index, static_cast<int64_t>(t) - 1, w);
    return lookback_finish<ROWS>(index, t, agg, bad, w, range_out);
}


// Ablation (NEXT #2): the plain chained scan that decoupled lookback replaces
// (Fig 12 left) — wait until the immediate predecessor holds its
// inclusive prefix, then publish this tile's.
__device__ __forceinline__ uint64_t chained_prefix(uint64_t *index, uint64_t t, uint64_t agg,
                                                   bool bad, bool *range_out) {
    const int lane = threadIdx.x & 31;
    uint64_t d = 0;
    if (lane == 0) {
        d = ld_relaxed_u64(&index[t - 1]);
        while ((d >> 62) != 2) {
            __nanosleep(32);
            d = ld_relaxed_u64(&index[t - 1]);
        }
    }
    d = __shfl_sync(0xffffffffu, d, 0);
    const uint64_t rbits = (d & BIT_RANGE) | (bad ? BIT_RANGE : 0);
    const uint64_t excl = d & VAL61;
    if (lane == 0) st_relaxed_u64(&index[t], FLAG_P | rbits | (excl + agg));
    *range_out = rbits != 0;
    return excl;
}

// ------------------------------------------------------------------ REL: min/max
__device__ __forceinline__ uint32_t sortable(float x) {
    uint32_t u = __float_as_uint(x);
    return u ^ ((u & 0x80000000u) ? 0xFFFFFFFFu : 0x80000000u);
}
__device__ __forceinline__ float unsortable(uint32_t u) {
    return __uint_as_float(u ^ ((u & 0x80000000u) ? 0x80000000u : 0xFFFFFFFFu));
}
__device__ __forceinline__ unsigned long long sortable(double x) {
    unsigned long long u = __double_as_longlong(x);
    return u ^ ((u >> 63) ? 0xFFFFFFFFFFFFFFFFull : 0x8000000000000000ull);
}
__device__ __forceinline__ double unsortable(unsigned long long u) {
    return __longlong_as_double(u ^ ((u >> 63) ? 0x8000000000000000ull : 0xFFFFFFFFFFFFFFFFull));
}

// Block reduction of (mn, mx), sortable-integer atomics into the header scratch, and
// the last CTA's finalisation: eb_abs = λ·(max − min) (R-15). Every thread calls it.
template <typename T>
__device__ __forceinline__ void minmax_finish(T mn, T mx, double lambda, uint8_t *__restrict__ hdr,
                                              double *__restrict__ range_out) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        mn = fmin(mn, __shfl_xor_sync(0xffffffffu, mn, o));
        mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    }
    __shared__ T s_mn[8], s_mx[8];
    __shared__ bool s_last;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (lane == 0) {
        s_mn[warp] = mn;
        s_mx[warp] = mx;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < (int)(blockDim.x / 32); w++) {
            mn = fmin(mn, s_mn[w]);
            mx = fmax(mx, s_mx[w]);
        }
        if (mn <= mx) {  // at least one non-NaN value
            if (sizeof(T) == 4) {
                atomicMax(reinterpret_cast<unsigned *>(hdr + 40), (unsigned)sortable(mx));
                atomicMax(reinterpret_cast<unsigned *>(hdr + 48), ~(unsigned)sortable(mn));
            } else {
                atomicMax(reinterpret_cast<unsigned long long *>(hdr + 40),
                          (unsigned long long)sortable(mx));
                atomicMax(reinterpret_cast<unsigned long long *>(hdr + 48),
                          ~(unsigned long long)sortable(mn));
            }
        }
        __threadfence();
        unsigned prev = atomicAdd(reinterpret_cast<unsigned *>(hdr + 56), 1u);
        s_last = (prev == gridDim.x - 1);
    }
    __syncthreads();
    if (s_last && threadIdx.x == 0) {
        __threadfence();
        double r = 0.0, dmn = INFINITY, dmx = -INFINITY;  // (+inf, -inf): no non-NaN value
        if (sizeof(T) == 4) {
            unsigned emx = atomicAdd(reinterpret_cast<unsigned *>(hdr + 40), 0u);
            unsigned emn = ~atomicAdd(reinterpret_cast<unsigned *>(hdr + 48), 0u);
            if (emx != 0u) {
                dmn = (double)unsortable(emn);
                dmx = (double)unsortable(emx);
                r = __dsub_rn(dmx, dmn);
            }
        } else {
            unsigned long long emx =
                atomicAdd(reinterpret_cast<unsigned long long *>(hdr + 40), 0ull);
            unsigned long long emn =
                ~atomicAdd(reinterpret_cast<unsigned long long *>(hdr + 48), 0ull);
            if (emx != 0ull) {
                dmn = unsortable(emn);
                dmx = unsortable(emx);
                r = __dsub_rn(dmx, dmn);
            }
        }
        if (range_out) {
            range_out[0] = dmn;
            range_out[1] = dmx;
        }
        const double eb_abs = (r == 0.0) ? lambda : __dmul_rn(lambda, r);
        *reinterpret_cast<double *>(hdr + 32) = eb_abs;
        reinterpret_cast<unsigned long long *>(hdr + 40)[0] = 0ull;
        reinterpret_cast<unsigned long long *>(hdr + 40)[1] = 0ull;
        reinterpret_cast<unsigned long long *>(hdr + 40)[2] = 0ull;
    }
}

// Header scratch while the REL reduction runs (the memset zeroed it; the last
// CTA restores zeros): [40] sortable max, [48] ~sortable min, [56] u32 CTA counter.
template <typename T>
__global__ void __launch_bounds__(256) minmax_kernel(const T *__restrict__ in, uint64_t n,
                                                     double lambda, uint8_t *__restrict__ hdr,
                                                     double *__restrict__ range_out) {
    using V = typename std::conditional<sizeof(T) == 4, float4, double2>::type;
    constexpr int PER = 16 / sizeof(T);
    T mn = INFINITY, mx = -INFINITY;
    const uint64_t nvec = n / PER;
    const V *vin = reinterpret_cast<const V *>(in);
    const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
    uint64_t i = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    // 4-way unrolled grid-stride loop (loads in flight before the min/max)
    for (; i + 3 * stride < nvec; i += 4 * stride) {
        V v[4];
#pragma unroll
        for (int u = 0; u < 4; u++) v[u] = __ldcs(vin + i + u * stride);
#pragma unroll
        for (int u = 0; u < 4; u++) {
            const T *e = reinterpret_cast<const T *>(&v[u]);
#pragma unroll
            for (int k = 0; k < PER; k++) {
                mn = fmin(mn, e[k]);
                mx = fmax(mx, e[k]);
            }
        }
    }
    for (; i < nvec; i += stride) {
        V v = __ldcs(vin + i);
        const T *e = reinterpret_cast<const T *>(&v);
#pragma unroll
        for (int k = 0; k < PER; k++) {
            mn = fmin(mn, e[k]);
            mx = fmax(mx, e[k]);
        }
    }
    if (blockIdx.x == 0 && threadIdx.x < n - nvec * PER) {
        T e = in[nvec * PER + threadIdx.x];
        mn = fmin(mn, e);
        mx = fmax(mx, e);
    }
    minmax_finish<T>(mn, mx, lambda, hdr, range_out);
}

// The same reduction with the field streamed through shared memory by 1D bulk TMA
// copies (MM_STAGES chunks of 16 KiB per CTA in flight; CTA c takes chunks c, c+G, ...,
// counted from the END of the field, so that the field's first ~100 MB — the tiles the
// compressor claims first, right after this pass — are the most recently read and still
// in the 126 MB L2):
// bulk copies keep ~128 KiB per SM in flight with no load instructions, which the
// register-staged loop above cannot (it tops out near 6.6 TB/s, this near the HBM read
// rate). d_in is 16-byte aligned (cszp2_compress contract); the bytes past the last
// whole chunk are read directly by CTA 0.
// Global REL: eb_abs = λ·(max − min) from a range the caller reduced
// across ranks (range[0] = min, range[1] = max as f64; min > max: no value), with the
// same arithmetic and zero-range rule as minmax_finish.
__global__ void eb_from_range_kernel(const double *__restrict__ range, double lambda,
                                     uint8_t *__restrict__ hdr) {
    const double mn = range[0], mx = range[1];
    const double r = (mn <= mx) ? __dsub_rn(mx, mn) : 0.0;
    *reinterpret_cast<double *>(hdr + 32) = (r == 0.0) ? lambda : __dmul_rn(lambda, r);
}

constexpr uint32_t MM_CHUNK = 16384;
constexpr int MM_STAGES = 4;
template <typename T>
__global__ void __launch_bounds__(256) minmax_kernel_tma(const T *__restrict__ in, uint64_t n,
                                                         double lambda, uint8_t *__restrict__ hdr,
                                                     double *__restrict__ range_out) {
    extern __shared__ __align__(128) uint8_t mm_smem[];
    __shared__ uint64_t s_full[MM_STAGES];
    using V = typename std::conditional<sizeof(T) == 4, float4, double2>::type;
    constexpr int PER = 16 / sizeof(T);
    const uint64_t nchunks = n * sizeof(T) / MM_CHUNK;
    const uint8_t *src = reinterpret_cast<const uint8_t *>(in);
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int k = 0; k < MM_STAGES; k++) mbar_init(&s_full[k], 1);
        fence_mbar_init();
        for (int k = 0; k < MM_STAGES; k++) {
            const uint64_t c = blockIdx.x + static_cast<uint64_t>(k) * gridDim.x;
            if (c < nchunks) {
                mbar_expect_tx(&s_full[k], MM_CHUNK);
                bulk_load(mm_smem + k * MM_CHUNK, src + (nchunks - 1 - c) * MM_CHUNK, MM_CHUNK, &s_full[k]);
            }
        }
    }
    __syncthreads();
    T mn = INFINITY, mx = -INFINITY;
    uint32_t it = 0;
    for (uint64_t c = blockIdx.x; c < nchunks; c += gridDim.x, ++it) {
        const int k = it % MM_STAGES;
        mbar_wait(&s_full[k], (it / MM_STAGES) & 1);
        const V *v = reinterpret_cast<const V *>(mm_smem + k * MM_CHUNK);
#pragma unroll
        for (int u = 0; u < (int)(MM_CHUNK / 16 / 256); u++) {
            const V w = v[u * 256 + tid];
            const T *e = reinterpret_cast<const T *>(&w);
#pragma unroll
            for (int j = 0; j < PER; j++) {
                mn = fmin(mn, e[j]);
                mx = fmax(mx, e[j]);
            }
        }
        __syncthreads();  // stage k consumed
        const uint64_t cn = c + static_cast<uint64_t>(MM_STAGES) * gridDim.x;
        if (tid == 0 && cn < nchunks) {
            mbar_expect_tx(&s_full[k], MM_CHUNK);
            bulk_load(mm_smem + k * MM_CHUNK, src + (nchunks - 1 - cn) * MM_CHUNK, MM_CHUNK, &s_full[k]);
        }
    }
    if (blockIdx.x == 0) {  // values past the last whole chunk
        for (uint64_t i = nchunks * (MM_CHUNK / sizeof(T)) + tid; i < n; i += blockDim.x) {
            mn = fmin(mn, in[i]);
            mx = fmax(mx, in[i]);
        }
    }
    minmax_finish<T>(mn, mx, lambda, hdr, range_out);
}

// ------------------------------------------------------------------ compression
struct HdrStatic {
    uint32_t word1;    // header bytes 4..7: version, dtype, enc_mode, log2L
    uint32_t eb_mode;  // header byte 8
    double eb_user;    // header bytes 24..31
    uint32_t flags;    // CSZP2_FLAG_* (ablations)
};

// Warp-specialised compression CTA (NT_COMP = 288 threads = 9 warps; 3 CTAs per SM
// for f32):
//   producers  warps 0-7  one thread per 32-value block. Thread 0 also claims
//                         tiles from the atomic ticket (in order, so every predecessor a
//                         lookback waits for belongs to a running CTA) and TMA-loads
//                         them, one tile ahead, into the single input buffer, which is
//                         free again as soon as the values are in registers. Per tile:
//                         encode (❶ ❷), publish the aggregate, stage the payload in a
//                         byte ring, queue it.
//   resolver   warp 8     for each queued tile, in order: decoupled lookback (❸), then
//                         copy its payload from the ring to its place (❹) and free the
//                         ring bytes and the queue slot; the last tile also writes
//                         pads, header and *d_out_bytes.
// The rule that keeps the GPU from serialising on the inclusive-prefix frontier: a
// claimed tile never waits on anything that depends on a lookback. The next tile is
// claimed ahead only while the ring clearly has room for two more payloads (so the
// producers do not block on the ring while holding it); otherwise it is claimed after
// the current tile is staged.
constexpr int NT_COMP = NT + 32;
constexpr int RESOLVE_WARP = NT / 32;  // warp 8
constexpr int NQ = 16;                 // queue slots (tiles staged ahead of the resolver)
constexpr uint32_t BAR_PROD = 1;

// The staging ring lives in a virtual byte space of RING_V per lap (a power of 2, so
// u32 cursors wrap consistently) of which the first RING bytes exist: an allocation
// never straddles RING (it moves to the next lap instead), so virtual position p is
// physical byte p % RING_V and the room test is pos + bytes <= tail + RING_V.
// 40 KiB: the most that keeps three f32 CTAs per SM (3 x (32 KiB tile + 40 KiB ring +
// alignment + static) <= 228 KiB; f64: two CTAs with 64 KiB tiles); at CR ~2.5 a tile
// stages ~14 KiB and stays in the ring for one lookback latency (~6 us at cfg4a), so
// the 32 KiB ring of round 1 held only two of them.
template <typename T>
struct CompLayout {
    static constexpr uint32_t IN_BYTES = Traits<T>::TILE_BYTES;  // one TMA tile
    static constexpr uint32_t RING = 40960;  // >= the largest tile payload (256 x 128 B)
    static constexpr uint32_t RING_V = 65536;
    static constexpr int SMEM = IN_BYTES + RING + 64 + 1024;
};
template <typename T>
constexpr int compress_smem_bytes() {
    return CompLayout<T>::SMEM;
}

// Copy a tile's staged payload (smem, 16-byte aligned base) to its global byte
// range [dst0, dst0 + bytes) with threads w = 0..nw-1: 16-byte aligned chunks by
// coalesced 128-bit stores (funnel-shifted out of smem), the unaligned head/tail by
// bytes (nw >= 32).
__device__ __forceinline__ void write_payload(const uint8_t *stg, uint8_t *out, uint64_t dst0,
                                              uint32_t bytes, int w, int nw) {
    const uint64_t dst1 = dst0 + bytes;
    const uint64_t a0 = roundup16(dst0), a1 = dst1 & ~uint64_t(15);
    if (a0 < a1) {
        const uint32_t s0 = static_cast<uint32_t>(a0 - dst0);  // 0..15
        const uint32_t sh = 8u * (s0 & 3u);
        const uint32_t *sw = reinterpret_cast<const uint32_t *>(stg) + (s0 >> 2);
        const uint32_t nchunks = static_cast<uint32_t>((a1 - a0) >> 4);
        for (uint32_t c = w; c < nchunks; c += nw) {
            const uint32_t *p = sw + 4 * c;
            const uint32_t v0 = p[0], v1 = p[1], v2 = p[2], v3 = p[3], v4 = p[4];
            uint4 o;
            o.x = __funnelshift_r(v0, v1, sh);
            o.y = __funnelshift_r(v1, v2, sh);
            o.z = __funnelshift_r(v2, v3, sh);
            o.w = __funnelshift_r(v3, v4, sh);
            *reinterpret_cast<uint4 *>(out + a0 + 16ull * c) = o;
        }
        if (w < 16) {  // head bytes
            const uint64_t o = dst0 + w;
            if (o < a0) out[o] = stg[o - dst0];
        } else if (w < 32) {  // tail bytes
            const uint64_t o = a1 + (w - 16);
            if (o < dst1) out[o] = stg[o - dst0];
        }
    } else if (w < 32) {  // the whole payload is < 32 bytes
        const uint64_t o = dst0 + w;
        if (o < dst1) out[o] = stg[o - dst0];
    }
}

// LOAD (NEXT #2 memory ablation, Fig 10-11): 0 = TMA tensor tiles (the
// product path), 1 = each thread reads its own block with 16-byte vector loads (the
// paper's vectorised access), 2 = each thread reads its block value by value.
constexpr int LOAD_TMA = 0, LOAD_VEC = 1, LOAD_SCALAR = 2;

template <typename T, bool OUTLIER, int LOAD = LOAD_TMA, int LBR = LB_PER_LANE>
__global__ void __launch_bounds__(NT_COMP, sizeof(T) == 4 ? 3 : 2) compress_kernel(
    const __grid_constant__ CUtensorMap tmap, const T *__restrict__ in, const Geom g,
    const double eb_abs_arg, const int eb_from_header, uint8_t *__restrict__ out,
    unsigned *__restrict__ ticket, uint64_t *__restrict__ d_out_bytes, const HdrStatic hs) {
    using LY = CompLayout<T>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t *inbuf = smem_align<1024>(smem_raw);
    uint8_t *ring = inbuf + LY::IN_BYTES;
    __shared__ uint64_t s_full;                    // input buffer
    __shared__ uint64_t s_staged[NQ], s_done[NQ];  // queue slots
    __shared__ uint64_t s_qt[NQ];
    __shared__ uint32_t s_qagg[NQ], s_qpos[NQ];
    __shared__ uint8_t s_qbad[NQ];
    __shared__ uint32_t s_warp[2][NT / 32];  // tile_scan_1bar, by tile parity
    __shared__ uint32_t s_tailb[2];          // s_tail as thread 0 acquired it before the scan, by tile parity
    __shared__ uint32_t s_tail;              // ring bytes released by the resolver
    __shared__ uint32_t s_tkin;
    __shared__ uint64_t s_rel;            // producer warps done reading the input buffer
    __shared__ volatile uint32_t s_end;   // queue index of the end marker

    const int tid = threadIdx.x;
    const int warp = tid >> 5;
    const uint64_t T_eff = g.T ? g.T : 1;
    uint64_t *index = reinterpret_cast<uint64_t *>(out + 64);
    const double eb_abs =
        eb_from_header ? *reinterpret_cast<const volatile double *>(out + 32) : eb_abs_arg;

    // producer thread 0: TMA-load tile tk into the input buffer (always arrives on
    // s_full so its phase advances even without data)
    auto issue = [&](uint64_t tk) {
        const uint64_t b0 = tk * BPT;
        if (LOAD == LOAD_TMA && b0 < g.nfull) {
            if (Traits<T>::ROWS == 1) {
                mbar_expect_tx(&s_full, BPT * 128);
                tma_load_2d_ef(inbuf, &tmap, 0, static_cast<int>(b0), &s_full);
            } else {
                const bool second = (b0 + BPT / 2) < g.nfull;
                mbar_expect_tx(&s_full, second ? 2 * BPT * 128 : BPT * 128);
                tma_load_2d_ef(inbuf, &tmap, 0, static_cast<int>(2 * b0), &s_full);
                if (second) tma_load_2d_ef(inbuf + BPT * 128, &tmap, 0, static_cast<int>(2 * b0 + BPT), &s_full);
            }
        } else {
            mbar_expect_tx(&s_full, 0);
        }
    };
    // producer thread 0: publish the claimed ticket, then arrive on s_full (with the
    // TMA bytes, or without data past the last tile): the mbarrier's release/acquire
    // makes s_tkin visible to the producers waiting on s_full, so no extra barrier
    auto claim = [&](uint32_t tk) {
        s_tkin = tk;
        if (tk < T_eff) {
            TRACE(tk, 0, gtimer());
            TRACE(tk, 7, blockIdx.x);
            issue(tk);
        } else {
            mbar_expect_tx(&s_full, 0);
        }
    };

    constexpr uint32_t RING = LY::RING, RING_V = LY::RING_V;
    for (uint32_t c = tid; c < RING / 16; c += NT_COMP)  // staging ring starts zeroed
        reinterpret_cast<uint4 *>(ring)[c] = make_uint4(0, 0, 0, 0);
    if (tid == 0) {
        s_end = 0xFFFFFFFFu;
        s_tail = 0;
        mbar_init(&s_rel, NT / 32);
        mbar_init(&s_full, 1);
        for (int i = 0; i < NQ; i++) {
            mbar_init(&s_staged[i], NT / 32);
            mbar_init(&s_done[i], 1);
        }
        fence_mbar_init();
        claim(atomicAdd(ticket, 1u));
    }
    __syncthreads();

    if (warp < RESOLVE_WARP) {
        // ============================== producers
        const auto K = make_consts(eb_abs, static_cast<T *>(nullptr));
        // ring allocation cursor and latest payload size: identical in every producer thread
        uint32_t head = 0, last_agg = 0;
        // where a payload of `bytes` would go, and whether it fits now
        auto place = [&](uint32_t bytes) {
            uint32_t pos = (head + 15u) & ~15u;
            if ((pos % RING_V) + bytes > RING) pos = (pos / RING_V + 1) * RING_V;
            return pos;
        };
        auto fits = [&](uint32_t pos, uint32_t bytes, uint32_t tl) { return pos + bytes <= tl + RING_V || tl == head; };
        for (uint32_t it = 0;; ++it) {
            const int q = it % NQ;
            // thread 0 takes the next ticket while the data is in flight if this tile's
            // payload (estimated from the last one) fits in the ring now, i.e. its staging
            // will not wait on a lookback while the ticket is held unpublished; the
            // atomic's result stays in a register until the buffer is released, so
            // nothing waits on its round trip
            uint32_t tk_next = 0;
            bool ahead = false;
            if (tid == 0) {
                // the ring's free cursor, acquired: the resolver's clears of the freed bytes
                // happen-before it, and the scan barrier hands it to every producer
                const uint32_t tl = ld_acquire_cta(&s_tail);
                s_tailb[it & 1] = tl;
                const uint32_t est = min(BPT * 4u * L, last_agg + last_agg / 4u + 256u);
                ahead = fits(place(est), est, tl);
                if (ahead) tk_next = atomicAdd(ticket, 1u);
            }
            mbar_wait(&s_full, it & 1);
            const uint64_t t = s_tkin;  // published before the arrival we just waited for
            if (t >= T_eff) {           // end marker for the resolver (one arrival per warp)
                if ((tid & 31) == 0) {
                    if (it >= NQ) mbar_wait(&s_done[q], (it / NQ - 1) & 1);  // slot free
                    if (tid == 0) s_end = it;
                    mbar_arrive(&s_staged[q]);
                }
                break;
            }
            if (tid == 0) TRACE(t, 1, gtimer());
            const uint64_t b = t * BPT + tid;
            const bool active = b < g.nb;
            const bool full = b < g.nfull;

            T x[L];
            uint32_t valid = L;
            if (full && LOAD == LOAD_TMA) {
                load_block(inbuf, tid, x);
            } else if (full && LOAD == LOAD_VEC) {
                const uint4 *src = reinterpret_cast<const uint4 *>(in + b * L);
#pragma unroll
                for (int v = 0; v < L * (int)sizeof(T) / 16; v++)
                    *reinterpret_cast<uint4 *>(reinterpret_cast<uint8_t *>(x) + 16 * v) = __ldg(src + v);
            } else if (full) {
#pragma unroll
                for (int i = 0; i < L; i++) x[i] = __ldg(in + b * L + i);
            } else {
                valid = active ? static_cast<uint32_t>(g.n - b * L) : 0u;
#pragma unroll
                for (int i = 0; i < L; i++) x[i] = (i < (int)valid) ? in[b * L + i] : T(0);
            }

            // The input buffer is free once every producer warp holds its values in
            // registers (s_rel: one arrival per warp): warp 0 then issues the TMA load of
            // the tile taken ahead (otherwise thread 0 claims after staging), so the load
            // overlaps this tile's whole encode; the other warps go straight on.
            __syncwarp();
            if ((tid & 31) == 0) mbar_arrive(&s_rel);
            if (warp == 0) {
                mbar_wait(&s_rel, it & 1);
                if (ahead) claim(tk_next);
            }

            // ❶ pre-quantization + in-block first-order difference
            bool bad = false;
            int qv[L];
            uint32_t a[L];
            uint32_t sign = 0, or_rest = 0;
            auto difference = [&]() {
                if (!full) {  // tail block: q_i = q_{i-1} past n (FORMAT.md §6.4)
#pragma unroll
                    for (int i = 1; i < L; i++)
                        if (i >= (int)valid) qv[i] = qv[i - 1];
                }
                sign = 0;
                or_rest = 0;
#pragma unroll
                for (int i = L - 1; i >= 0; i--) {
                    // biased patterns difference to d_i (mod 2^32; |d_i| < 2^31 by the range check)
                    const int d = static_cast<int>(static_cast<uint32_t>(qv[i]) -
                                                   static_cast<uint32_t>(i ? qv[i - 1] : QBias<T>::value));
                    a[i] = static_cast<uint32_t>(d < 0 ? -d : d);
                    sign = __funnelshift_l(static_cast<uint32_t>(d), sign, 1);  // bit i = d_i < 0
                    if (i) or_rest |= a[i];
                }
            };
            if constexpr (sizeof(T) == 4) {
                // unchecked patterns first; a block they may not cover exactly (fl_p > 17,
                // see quantize_block_unchecked) is redone with the checked quantizer
                quantize_block_unchecked(x, K.inv, qv);
                difference();
                if (32 - __clz(or_rest | a[0]) > FAST_FL_MAX) {
                    // rare: re-read the block from global memory (x is dead by now, and
                    // keeping it live would cost registers on the common path)
#pragma unroll
                    for (int i = 0; i < L; i++) x[i] = (i < (int)valid) ? in[b * L + i] : T(0);
                    quantize_block(x, K.inv, qv, bad);
                    difference();
                }
            } else {
                quantize_block(x, K.inv, qv, bad);
                difference();
            }

            // ❷ fixed lengths and the fine-tuned Plain/Outlier selection
            const int fl_p = 32 - __clz(or_rest | a[0]);
            uint32_t size = fl_p ? 4u * (1u + fl_p) : 0u;
            uint32_t obyte = static_cast<uint32_t>(fl_p);
            int fl = fl_p, nob = 0;
            if (OUTLIER) {
                const int fl_o = 32 - __clz(or_rest);
                const int ob = max(1, (32 - __clz(a[0]) + 7) >> 3);
                const uint32_t size_o = 4u + ob + 4u * fl_o;
                if (size_o < size) {
                    size = size_o;
                    obyte = 0x80u | (static_cast<uint32_t>(ob - 1) << 5) | static_cast<uint32_t>(fl_o);
                    fl = fl_o;
                    nob = ob;
                }
            }
            if (!active) {
                size = 0;
                bad = false;
            }
            if (!K.ok) bad = true;

            // intra-tile scan ("Reduce") and the tile's range flag, one barrier
            uint32_t agg;
            bool any_bad;
            const uint32_t my_excl = tile_scan_1bar(size, bad, s_warp[it & 1], &agg, &any_bad, BAR_PROD);
            if (tid == 0 && g.T) publish_aggregate(index, t, agg, any_bad);
            if (tid == 0) TRACE(t, 2, gtimer());
            // ring space (16-aligned, contiguous), computed identically by every producer
            // thread from (head, agg); each waits for room itself. An empty ring always has
            // room (a payload that had to skip the ring's end can then never find the
            // skipped bytes still "in use").
            // room with thread 0's acquired free cursor (bar.sync orders that acquire before
            // every producer's staging stores); else each thread spins with acquire loads
            const uint32_t pos = place(agg);
            if (!fits(pos, agg, s_tailb[it & 1]))
                while (!fits(pos, agg, ld_acquire_cta(&s_tail))) __nanosleep(64);
            head = pos + agg;
            last_agg = agg;
            if (active) out[g.O + b] = static_cast<uint8_t>(obyte);  // ❹ offset bytes

            // ❷ payload staged in the ring at its tile-relative byte offset; bit planes
            // by an in-register transpose sized to the warp's largest fixed length
            {
                const uint32_t st = (pos % RING_V) + my_excl;
                const uint32_t outl = a[0];
                if (OUTLIER && nob) a[0] = 0;  // the outlier slot of every plane is 0
                const int flw = static_cast<int>(__reduce_max_sync(0xffffffffu, static_cast<unsigned>(size ? fl : 0)));
                if (size) {
                    if (flw == 0) {  // only headers (Outlier blocks with fl = 0): no planes
                        stage_payload<0>(ring, st, sign, outl, nob, 0, a);
                    } else if (flw <= 1) {
                        pack_planes<0>(a);
                        stage_payload<1>(ring, st, sign, outl, nob, fl, a);
                    } else if (flw <= 2) {
                        pack_planes<1>(a);
                        stage_payload<2>(ring, st, sign, outl, nob, fl, a);
                    } else if (flw <= 4) {
                        pack_planes<2>(a);
                        stage_payload<4>(ring, st, sign, outl, nob, fl, a);
                    } else if (flw <= 8) {
                        pack_planes<3>(a);
                        stage_payload<8>(ring, st, sign, outl, nob, fl, a);
                    } else if (flw <= 16) {
                        pack_planes<4>(a);
                        stage_payload<16>(ring, st, sign, outl, nob, fl, a);
                    } else {
                        pack_planes<5>(a);
                        stage_payload<32>(ring, st, sign, outl, nob, fl, a);
                    }
                }
            }
            // this warp's blocks are staged: one arrival per warp on the queue slot (no
            // CTA barrier — a warp with nothing to stage goes on to the next tile);
            // thread 0 fills in the slot first. Every arriving warp waits for the slot
            // to be free, so s_staged[q] never runs a phase ahead of the resolver.
            __syncwarp();
            if ((tid & 31) == 0) {
                if (it >= NQ) mbar_wait(&s_done[q], (it / NQ - 1) & 1);  // queue slot free
                if (tid == 0) {
                    TRACE(t, 4, gtimer());
                    s_qt[q] = t;
                    s_qagg[q] = agg;
                    s_qbad[q] = any_bad;
                    s_qpos[q] = pos;
                }
                mbar_arrive(&s_staged[q]);
            }
            // claim now: nothing unpublished is held, and the claimed tile publishes its
            // aggregate before it can wait for ring room, so no wait is needed here
            if (tid == 0 && !ahead) claim(atomicAdd(ticket, 1u));
        }
    } else {
        // ============================== resolver: ❸ then ❹, in tile order
        // (Issuing the next queued tile's lookback window before this tile's copy was
        // measured 5-13% slower: the early snapshot holds Waiting descriptors that have
        // published by the time it is read, and every one costs a back-off re-poll.)
        const int lane = tid & 31;
        const bool chained = (hs.flags & 1u) != 0;
        for (uint32_t it = 0;; ++it) {
            const int q = it % NQ;
            mbar_wait_backoff(&s_staged[q], (it / NQ) & 1, 100);
            if (it >= s_end) break;
            const uint64_t t = s_qt[q];
            const uint32_t agg = s_qagg[q];
            const uint32_t pos = s_qpos[q];
            const bool bad = s_qbad[q];
            if (lane == 0) TRACE(t, 6, gtimer());
            bool rng = bad;
            uint64_t excl = 0;
            if (lane == 0) TRACE(t, 8, gtimer());
            if (g.T && t > 0) {
                if (chained)  // ablation: plain chained scan (Fig 12 left)
                    excl = chained_prefix(index, t, agg, bad, &rng);
                else
                    excl = lookback<LBR>(index, t, agg, bad, &rng);
            }
            if (lane == 0) TRACE(t, 3, gtimer());
            const uint64_t dst0 = g.D + excl;
            write_payload(ring + (pos % RING_V), out, dst0, agg, lane, 32);
            if (lane == 0) TRACE(t, 9, gtimer());
            if (t == T_eff - 1) {  // last tile: pads, header, d_out_bytes
                const uint64_t dst1 = dst0 + agg;
                __syncwarp();
                if (lane < 16) {  // zero pad after the payload
                    const uint64_t o = dst1 + lane;
                    if (o < roundup16(dst1)) out[o] = 0;
                } else {  // zero pad after the offset bytes
                    const uint64_t o = g.O + g.nb + (lane - 16);
                    if (o < g.D) out[o] = 0;
                }
                if (lane == 0) {
                    const uint32_t status = rng ? ST_RANGE : 0u;
                    const uint64_t pb = status ? 0 : excl + agg;
                    const uint64_t total = roundup16(g.D + pb);
                    uint64_t *h = reinterpret_cast<uint64_t *>(out);
                    h[0] = MAGIC | (static_cast<uint64_t>(hs.word1) << 32);
                    h[1] = hs.eb_mode | (status << 8) | (static_cast<uint64_t>(BPT) << 16);
                    h[2] = g.n;
                    h[3] = static_cast<uint64_t>(__double_as_longlong(hs.eb_user));
                    h[4] = static_cast<uint64_t>(__double_as_longlong(eb_abs));
                    h[5] = pb;
                    h[6] = total;
                    h[7] = 0;
                    if (d_out_bytes) *d_out_bytes = total;
                }
            }
            __syncwarp();  // every lane is done reading these ring bytes: clear them for reuse
            {
                uint4 *z = reinterpret_cast<uint4 *>(ring + (pos % RING_V));
                for (uint32_t c = lane; c < (agg + 15u) / 16u; c += 32) z[c] = make_uint4(0, 0, 0, 0);
            }
            __syncwarp();  // every lane's zero stores are ordered before lane 0's release below
            if (lane == 0) {
                __threadfence_block();  // release pattern: fence, then the relaxed cursor store
                st_relaxed_cta(&s_tail, pos + agg);  // in order, so the ring frees in order
                mbar_arrive(&s_done[q]);
            }
        }
    }
}

// ------------------------------------------------------------------ block decode
// ❷⁻¹ + inverse Lorenzo + ❶⁻¹ of one block whose payload starts at byte `pos` of the
// shared buffer `pbuf`: sign field, outlier, bit planes (in-register
// transpose sized to the warp's largest fixed length), q_i = q_{i-1} + d_i,
// x_i = (T)q_i * s. Warp-collective: every lane of the warp must call it.
template <typename T>
__device__ __forceinline__ void decode_block(const uint8_t *pbuf, uint32_t pos, uint32_t obyte,
                                             uint32_t size, T s, T (&x)[L]) {
    const uint32_t fl = obyte & 31u;
    const bool is_o = (obyte & 0x80u) != 0;
    const uint32_t nob = is_o ? ((obyte >> 5) & 3u) + 1u : 0u;
    uint32_t a[L];
    uint32_t sign = 0, outlier = 0;
    const int flw = static_cast<int>(__reduce_max_sync(0xffffffffu, size ? fl : 0u));
    if (size) {
        sign = ld_u32_unaligned(pbuf, pos);
        pos += 4;
        if (is_o) {
            outlier = ld_u32_unaligned(pbuf, pos);
            if (nob < 4) outlier &= (1u << (8 * nob)) - 1u;
            pos += nob;
        }
    }
    // every row of a[] is written once: zeros, or load_planes (rows < R; a block with
    // size 0 has fl 0, so its planes load as zeros) + unpack_planes (rows >= R)
    if (flw == 0) {
#pragma unroll
        for (int i = 0; i < L; i++) a[i] = 0;
    } else {
        if (flw <= 1) {
            load_planes<1>(pbuf, pos, fl, a);
            unpack_planes<0>(a);
        } else if (flw <= 2) {
            load_planes<2>(pbuf, pos, fl, a);
            unpack_planes<1>(a);
        } else if (flw <= 4) {
            load_planes<4>(pbuf, pos, fl, a);
            unpack_planes<2>(a);
        } else if (flw <= 8) {
            load_planes<8>(pbuf, pos, fl, a);
            unpack_planes<3>(a);
        } else if (flw <= 16) {
            load_planes<16>(pbuf, pos, fl, a);
            unpack_planes<4>(a);
        } else {
            load_planes<32>(pbuf, pos, fl, a);
            unpack_planes<5>(a);
        }
    }
    if (is_o) a[0] = outlier;
    int qv = 0;
#pragma unroll
    for (int i = 0; i < L; i++) {
        const int d = ((sign >> i) & 1u) ? -static_cast<int>(a[i]) : static_cast<int>(a[i]);
        qv += d;
        x[i] = dequantize(qv, s);
    }
}

// Header checks shared by the decompression kernels (FORMAT.md §3): returns 0, or
// ST_FORMAT / ST_RANGE; *eb and *pb receive eb_abs and the payload byte count.
template <typename T>
__device__ __forceinline__ int check_header(const uint8_t *cmp, const Geom &g, double *eb,
                                            uint64_t *pb) {
    const uint64_t *h = reinterpret_cast<const uint64_t *>(cmp);
    const uint64_t h0 = h[0], h1 = h[1];
    int err = 0;
    const uint32_t want1 = 1u | (static_cast<uint32_t>(Traits<T>::DTYPE) << 8) | (5u << 24);
    if ((h0 & 0xFFFFFFFFu) != MAGIC || ((h0 >> 32) & 0xFF00FFFFu) != want1 ||
        ((h1 >> 16) & 0xFFFFu) != BPT || (h1 >> 32) != 0 /* 1D predictor, FORMAT.md §7 */ ||
        h[2] != g.n)
        err = ST_FORMAT;
    else if (((h1 >> 8) & 0xFF) != 0)
        err = ((h1 >> 8) & 0xFF) == ST_RANGE ? ST_RANGE : ST_FORMAT;
    *pb = h[5];
    if (!err && h[6] != roundup16(g.D + *pb)) err = ST_FORMAT;
    *eb = __longlong_as_double(static_cast<long long>(h[4]));
    return err;
}

// ------------------------------------------------------------------ decompression
constexpr uint32_t PBUF_BYTES = BPT * 4 * L + 128;  // max tile payload + alignment slack

template <typename T>
constexpr int decompress_smem_bytes() {
    return Traits<T>::TILE_BYTES + PBUF_BYTES + 1024;
}

// Persistent decompression kernel: CTA c decodes tiles c, c+G, c+2G, ... The
// persisted tile index locates every tile in O(1) (no inter-CTA waiting), so the
// next tile's index words, offset bytes and payload (1D bulk TMA) are fetched
// while the current tile is decoded and stored (2D tensor TMA, 128B swizzle).
// Payloads land in one 32 KiB ring, the next tile's right behind the current one
// (at useful compression ratios both fit, so the fetch overlaps the decode); only
// when they do not is the fetch deferred until the current tile is decoded. One
// payload buffer instead of two fits three CTAs per SM for f32.
template <typename T>
__global__ void __launch_bounds__(NT, sizeof(T) == 4 ? 3 : 2) decompress_kernel(const __grid_constant__ CUtensorMap tmap,
                                                           const uint8_t *__restrict__ cmp,
                                                           T *__restrict__ out, const Geom g,
                                                           int *__restrict__ d_status) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t *ostage = smem_align<1024>(smem_raw);
    uint8_t *ring = ostage + Traits<T>::TILE_BYTES;
    __shared__ uint64_t s_bar[2];
    __shared__ uint32_t s_warp[NT / 32];
    __shared__ uint64_t s_excl[2];
    __shared__ uint32_t s_bytes[2];
    __shared__ uint32_t s_rpos[2];  // ring position of each slot's payload
    __shared__ double s_eb;
    __shared__ int s_err;

    const int tid = threadIdx.x;
    const uint64_t G = gridDim.x;
    const uint64_t *index = reinterpret_cast<const uint64_t *>(cmp) + 8;
    constexpr uint32_t BAD_BYTES = 0xFFFFFFFFu;

    // thread 0 state: raw index words of the tile two steps ahead
    uint64_t raw_p = FLAG_P, raw_i = 0;
    uint64_t pb_hdr = 0;   // payload bytes from the header
    bool pending = false;  // a payload prefetch is in flight

    // thread 0 ring state: [r_pos, r_pos + r_len) holds the current slot's payload
    uint32_t r_pos = 0, r_len = 0;
    bool deferred = false;  // next slot's payload waits for the ring to empty

    // thread 0: tile meta from two index words -> smem slot; start its payload TMA
    // into the ring (behind the current payload, else at 0 if that end is free) or
    // defer it (returns false) when neither fits yet.
    auto launch = [&](uint64_t dp, uint64_t di, int bi, bool ring_empty) -> bool {
        const uint64_t e = dp & VAL_MASK, i = di & VAL_MASK;  // bit 61 is 0 in a valid stream
        uint32_t bytes = BAD_BYTES;
        if ((dp >> 61) == 4 && (di >> 61) == 4 && i >= e && i <= pb_hdr &&
            i - e <= static_cast<uint64_t>(BPT) * 4 * L)
            bytes = static_cast<uint32_t>(i - e);
        s_excl[bi] = e;
        s_bytes[bi] = bytes;
        if (bytes != BAD_BYTES && bytes) {
            const uint64_t src0 = (g.D + e) & ~uint64_t(15);
            const uint32_t len = static_cast<uint32_t>(roundup16(g.D + e + bytes) - src0);
            uint32_t pos;
            if (ring_empty)
                pos = 0;
            else if (r_pos + r_len + len <= PBUF_BYTES - 16)
                pos = r_pos + r_len;
            else if (len + 16 <= r_pos)
                pos = 0;
            else
                return false;
            s_rpos[bi] = pos;
            r_pos = pos;
            r_len = len;
            mbar_expect_tx(&s_bar[bi], len);
            bulk_load(ring + pos, cmp + src0, len, &s_bar[bi]);
        } else {
            s_rpos[bi] = 0;
            r_len = 0;
            mbar_expect_tx(&s_bar[bi], 0);
        }
        return true;
    };

    uint64_t t = blockIdx.x;
    if (tid == 0) {
        // header checks (FORMAT.md §3) — once per CTA
        double eb;
        int err = check_header<T>(cmp, g, &eb, &pb_hdr);
        s_eb = eb;
        s_err = err;
        mbar_init(&s_bar[0], 1);
        mbar_init(&s_bar[1], 1);
        fence_mbar_init();
        if (!err && t < g.T) {
            launch(t ? index[t - 1] : FLAG_P, index[t], 0, true);
            pending = true;
            const uint64_t t2 = t + G;
            if (t2 < g.T) {
                raw_p = index[t2 - 1];
                raw_i = index[t2];
            }
        }
    }
    __syncthreads();
    if (s_err) {
        if (tid == 0 && d_status) atomicOr(d_status, s_err);
        return;
    }
    const auto K = make_consts(s_eb, static_cast<T *>(nullptr));
    uint32_t ob_cur = 0, ob_next = 0;
    {
        const uint64_t b = t * BPT + tid;
        if (t < g.T && b < g.nb) ob_cur = cmp[g.O + b];
        const uint64_t bn = (t + G) * BPT + tid;
        if (t + G < g.T && bn < g.nb) ob_next = cmp[g.O + bn];
    }

    int err = 0;
    for (uint32_t it = 0; t < g.T; ++it, t += G) {
        const int cur = it & 1;
        const uint64_t tn = t + G;
        uint64_t nraw_p = 0, nraw_i = 0;  // thread 0: the next tile's words if deferred
        if (tid == 0) {
            pending = false;
            deferred = false;
            if (tn < g.T) {  // payload of the next tile streams in during this one
                nraw_p = raw_p;
                nraw_i = raw_i;
                deferred = !launch(raw_p, raw_i, cur ^ 1, false);
                pending = !deferred;
                const uint64_t t2 = tn + G;
                if (t2 < g.T) {
                    raw_p = index[t2 - 1];
                    raw_i = index[t2];
                }
            }
        }
        uint32_t ob_pref = 0;  // offset byte of tile t + 2G, consumed two steps later
        {
            const uint64_t t2 = tn + G;
            const uint64_t b2 = t2 * BPT + tid;
            if (t2 < g.T && b2 < g.nb) ob_pref = cmp[g.O + b2];
        }

        const uint64_t b0 = t * BPT;
        const uint64_t b = b0 + tid;
        const bool active = b < g.nb;
        const uint32_t obyte = ob_cur;
        const uint32_t fl = obyte & 31u;
        const bool is_o = (obyte & 0x80u) != 0;
        const uint32_t nob = is_o ? ((obyte >> 5) & 3u) + 1u : 0u;
        const bool bad = (!is_o && (obyte & 0x60u));
        const uint32_t size = is_o ? 4u + nob + 4u * fl : (fl ? 4u * (1u + fl) : 0u);
        // one-barrier scan (+ OR of bad): s_warp is next rewritten after the two CTA
        // barriers below, so it needs no second barrier and no double buffer
        uint32_t agg;
        bool any_bad;
        const uint32_t my_excl = tile_scan_1bar(size, bad, s_warp, &agg, &any_bad, 0);
        if (any_bad || agg != s_bytes[cur]) {
            err = ST_FORMAT;
            if (tid == 0) {
                mbar_wait(&s_bar[cur], (it >> 1) & 1);
                if (pending) mbar_wait(&s_bar[cur ^ 1], ((it + 1) >> 1) & 1);
            }
            break;
        }
        mbar_wait(&s_bar[cur], (it >> 1) & 1);

        // ---- ❷⁻¹ decode, inverse Lorenzo, ❶⁻¹ dequantization
        T x[L];
        decode_block(ring + s_rpos[cur],
                     static_cast<uint32_t>((g.D + s_excl[cur]) & 15u) + my_excl, obyte, size, K.s, x);
        if (tid == 0) bulk_wait_read0();  // the previous tile's store has read ostage
        __syncthreads();
        if (tid == 0 && deferred) {  // the ring is empty now: fetch the next payload
            launch(nraw_p, nraw_i, cur ^ 1, true);
            pending = true;
        }
        const bool full = b < g.nfull;
        if (full) {
            store_block(ostage, tid, x);
        } else if (active) {  // ragged tail block: only valid values
            const uint32_t valid = static_cast<uint32_t>(g.n - b * L);
#pragma unroll
            for (int i = 0; i < L; i++)
                if (i < (int)valid) out[b * L + i] = x[i];
        }
        fence_proxy_async_smem();
        __syncthreads();
        if (tid == 0 && b0 < g.nfull) {
            if (Traits<T>::ROWS == 1) {
                tma_store_2d(&tmap, 0, static_cast<int>(b0), ostage);
            } else {
                tma_store_2d_ef(&tmap, 0, static_cast<int>(2 * b0), ostage);
                if (b0 + BPT / 2 < g.nfull)
                    tma_store_2d_ef(&tmap, 0, static_cast<int>(2 * b0 + BPT), ostage + BPT * 128);
            }
            bulk_commit();
        }
        ob_cur = ob_next;
        ob_next = ob_pref;
    }
    if (tid == 0) {
        bulk_wait_read0();
        if (err && d_status) atomicOr(d_status, err);
    }
}

// ------------------------------------------------------------------ random access
// Random-access decompression (§VI-B): values [first, first + count) of the
// stream, written to out[0 .. count). One CTA per tile covering the range; each tile is
// located in O(1) from the persisted index (R-14), so no scan over earlier tiles runs.
template <typename T>
__global__ void __launch_bounds__(NT) decompress_range_kernel(const uint8_t *__restrict__ cmp,
                                                              T *__restrict__ out, const Geom g,
                                                              uint64_t first, uint64_t count,
                                                              uint64_t t_begin,
                                                              int *__restrict__ d_status) {
    __shared__ __align__(16) uint8_t pbuf[PBUF_BYTES];
    __shared__ uint64_t s_bar;
    __shared__ uint32_t s_warp[NT / 32];
    __shared__ uint64_t s_excl;
    __shared__ uint32_t s_bytes;
    __shared__ double s_eb;
    __shared__ int s_err;
    const int tid = threadIdx.x;
    const uint64_t t = t_begin + blockIdx.x;
    if (tid == 0) {
        double eb;
        uint64_t pb;
        int err = check_header<T>(cmp, g, &eb, &pb);
        uint64_t e = 0, i = 0;
        if (!err) {
            const uint64_t *index = reinterpret_cast<const uint64_t *>(cmp) + 8;
            const uint64_t dp = t ? index[t - 1] : FLAG_P, di = index[t];
            e = dp & VAL_MASK;
            i = di & VAL_MASK;
            if ((dp >> 61) != 4 || (di >> 61) != 4 || i < e || i > pb ||
                i - e > static_cast<uint64_t>(BPT) * 4 * L)
                err = ST_FORMAT;
        }
        s_err = err;
        s_eb = eb;
        s_excl = e;
        s_bytes = static_cast<uint32_t>(i - e);
        mbar_init(&s_bar, 1);
        fence_mbar_init();
        if (!err) {
            if (i > e) {
                const uint64_t src0 = (g.D + e) & ~uint64_t(15);
                const uint32_t len = static_cast<uint32_t>(roundup16(g.D + i) - src0);
                mbar_expect_tx(&s_bar, len);
                bulk_load(pbuf, cmp + src0, len, &s_bar);
            } else {
                mbar_expect_tx(&s_bar, 0);
            }
        }
    }
    __syncthreads();
    if (s_err) {
        if (tid == 0 && d_status) atomicOr(d_status, s_err);
        return;
    }
    const uint64_t b = t * BPT + tid;
    const bool active = b < g.nb;
    const uint32_t obyte = active ? cmp[g.O + b] : 0u;
    const uint32_t fl = obyte & 31u;
    const bool is_o = (obyte & 0x80u) != 0;
    const uint32_t nob = is_o ? ((obyte >> 5) & 3u) + 1u : 0u;
    bool bad = (!is_o && (obyte & 0x60u));
    const uint32_t size = is_o ? 4u + nob + 4u * fl : (fl ? 4u * (1u + fl) : 0u);
    uint32_t agg;
    const uint32_t my_excl = cta_exclusive_scan(size, s_warp, &agg);
    bad |= (tid == 0 && agg != s_bytes);
    const bool any_bad = __syncthreads_or(bad);
    mbar_wait(&s_bar, 0);
    if (any_bad) {
        if (tid == 0 && d_status) atomicOr(d_status, ST_FORMAT);
        return;
    }
    const auto K = make_consts(s_eb, static_cast<T *>(nullptr));
    T x[L];
    decode_block(pbuf, static_cast<uint32_t>((g.D + s_excl) & 15u) + my_excl, obyte, size, K.s, x);
    const uint64_t v0 = b * L, last = first + count;
#pragma unroll
    for (int i = 0; i < L; i++) {
        const uint64_t v = v0 + i;
        if (v >= first && v < last && v < g.n) out[v - first] = x[i];
    }
}

// Ablation (NEXT #2): one CTA per tile in ticket order. LOOKBACK = the paper's
// decompression-side ❸: the tile's payload bytes are recomputed from its offset
// bytes, then a decoupled lookback over the scratch descriptors gives the tile's payload
// start. !LOOKBACK = the same kernel reading the start from the persisted tile index
// (R-14), so the two differ only in how the tile is located.
template <typename T, bool LOOKBACK>
__global__ void __launch_bounds__(NT) decompress_tilewise_kernel(const uint8_t *__restrict__ cmp,
                                                                 T *__restrict__ out, const Geom g,
                                                                 uint64_t *__restrict__ scratch,
                                                                 int *__restrict__ d_status) {
    __shared__ __align__(16) uint8_t pbuf[PBUF_BYTES];
    __shared__ uint64_t s_bar;
    __shared__ uint32_t s_warp[NT / 32];
    __shared__ uint64_t s_excl;
    __shared__ double s_eb;
    __shared__ int s_err;
    __shared__ uint32_t s_tk;
    const int tid = threadIdx.x;
    unsigned *ticket = reinterpret_cast<unsigned *>(scratch + (g.T ? g.T : 1));
    if (tid == 0) {
        s_tk = atomicAdd(ticket, 1u);
        double eb;
        uint64_t pb;
        s_err = check_header<T>(cmp, g, &eb, &pb);
        s_eb = eb;
        mbar_init(&s_bar, 1);
        fence_mbar_init();
    }
    __syncthreads();
    const uint64_t t = s_tk;
    // every CTA publishes (also on error) so no successor waits forever
    const uint64_t b = t * BPT + tid;
    const bool active = b < g.nb && !s_err;
    const uint32_t obyte = active ? cmp[g.O + b] : 0u;
    const uint32_t fl = obyte & 31u;
    const bool is_o = (obyte & 0x80u) != 0;
    const uint32_t nob = is_o ? ((obyte >> 5) & 3u) + 1u : 0u;
    bool bad = (!is_o && (obyte & 0x60u));
    const uint32_t size = is_o ? 4u + nob + 4u * fl : (fl ? 4u * (1u + fl) : 0u);
    uint32_t agg;
    const uint32_t my_excl = cta_exclusive_scan(size, s_warp, &agg);
    const bool any_bad = __syncthreads_or(bad);
    if (tid < 32) {
        uint64_t e = 0;
        bool rng = false;
        if (LOOKBACK) {
            if (tid == 0) publish_aggregate(scratch, t, agg, false);
            __syncwarp();
            if (t > 0) e = lookback(scratch, t, agg, false, &rng);
        } else if (t > 0 && t < g.T && !s_err) {
            const uint64_t d = reinterpret_cast<const uint64_t *>(cmp)[8 + t - 1];
            e = d & VAL_MASK;
        }
        if (tid == 0) {
            s_excl = e;
            if (!s_err && !any_bad && agg > 0) {
                const uint64_t src0 = (g.D + e) & ~uint64_t(15);
                const uint32_t len = static_cast<uint32_t>(roundup16(g.D + e + agg) - src0);
                mbar_expect_tx(&s_bar, len);
                bulk_load(pbuf, cmp + src0, len, &s_bar);
            } else {
                mbar_expect_tx(&s_bar, 0);
            }
        }
    }
    __syncthreads();
    if (s_err || any_bad) {
        if (tid == 0 && d_status) atomicOr(d_status, s_err ? s_err : ST_FORMAT);
        return;
    }
    mbar_wait(&s_bar, 0);
    const auto K = make_consts(s_eb, static_cast<T *>(nullptr));
    T x[L];
    decode_block(pbuf, static_cast<uint32_t>((g.D + s_excl) & 15u) + my_excl, obyte, size, K.s, x);
    if (b < g.nfull) {
        uint4 *dst = reinterpret_cast<uint4 *>(out + b * L);
#pragma unroll
        for (int v = 0; v < L * (int)sizeof(T) / 16; v++)
            dst[v] = *reinterpret_cast<const uint4 *>(reinterpret_cast<const uint8_t *>(x) + 16 * v);
    } else if (b < g.nb) {
#pragma unroll
        for (int i = 0; i < L; i++)
            if (b * L + i < g.n) out[b * L + i] = x[i];
    }
}

// ------------------------------------------------------------------ encode scratch
// Zero `words` u64 from `p` (the header and/or the tile index = the lookback
// descriptors, FORMAT.md §2) and the 16-byte tile ticket, in one launch.
__global__ void zero_scratch_kernel(uint64_t *__restrict__ p, uint64_t words, uint4 *__restrict__ ticket) {
    const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
    for (uint64_t i = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < words; i += stride)
        p[i] = 0;
    if (blockIdx.x == 0 && threadIdx.x == 0) *ticket = make_uint4(0, 0, 0, 0);
}

// ------------------------------------------------------------------ container index
__global__ void container_index_kernel(const uint64_t *__restrict__ sizes, int nparts,
                                       uint64_t *__restrict__ offsets) {
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        uint64_t s = 0;
        for (int r = 0; r < nparts; r++) {
            offsets[r] = s;
            s += sizes[r];
        }
        offsets[nparts] = s;
    }
}

}  // namespace cszp2
