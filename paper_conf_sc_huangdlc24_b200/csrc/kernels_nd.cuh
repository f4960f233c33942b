// kernels_nd.cuh — NEXT #3: the multi-dimensional Lorenzo variants of the paper's
// §VI-D / Table VI: 2D Lorenzo on 8x8 blocks and 3D Lorenzo on 4x4x4
// blocks (L = 64), same Plain/Outlier FLE, same decoupled-lookback concatenation
// (FORMAT.md §7). The paper keeps them out of the main design because they cost
// throughput (>50%). Compression: warp-specialised persistent CTAs (8 producer
// warps, one thread per 64-value block, values gathered straight from global memory by
// 16-byte rows and quantized with the 1D kernel's unchecked magic-add under a per-block
// certificate; separable Lorenzo; 1 resolver warp for lookback + copy-out) claiming tiles
// in order from an atomic ticket. Decompression: f32 — persistent CTAs with the payload
// ring prefetch of the 1D kernel and row-by-row inverse Lorenzo + stores; f64 — one CTA
// per tile (decompress_nd_tile_kernel). DESIGN.md §6.
#pragma once
#include "kernels.cuh"

namespace cszp2 {

constexpr int LND = 64;  // values per multi-dimensional block

// Exact u32 division by a runtime constant for dividends < 2^31 (round-up multiplier,
// Granlund & Montgomery): q = umulhi(n, m) >> s, with m = ceil(2^(31+l) / d),
// l = ceil(log2 d); d = 1 is the identity (m = 0).
struct FastDiv {
    uint32_t d, m, s;
};
__host__ __device__ inline FastDiv make_fastdiv(uint32_t d) {
    FastDiv f{d, 0u, 0u};
    if (d > 1) {
        uint32_t l = 0;
        while ((1ull << l) < d) l++;
        const uint32_t p = 31 + l;
        f.m = static_cast<uint32_t>(((1ull << p) + d - 1) / d);
        f.s = p - 32;
    }
    return f;
}
__device__ __forceinline__ uint32_t fast_div(uint32_t n, const FastDiv &f) {
    return f.d == 1 ? n : (__umulhi(n, f.m) >> f.s);
}

struct GeomND {
    uint64_t nx, ny, nz;    // field extents, x fastest
    uint64_t nbx, nby, nbz; // block grid
    uint64_t n, nb, T, O, D;
    FastDiv dbx, dby;       // division by nbx, nby (used while nb < 2^31)
    uint64_t roff[16];      // compression gathers: byte offset of block row r (r = iy + BY iz)
    uint64_t ystep, zstep;  // the same as steps: row r-1 -> r within / across a z-plane
    uint32_t vec;           // rows are whole 16-byte vectors (nx % (16/w) == 0)
    uint32_t vec32;         // rows start 32-byte aligned (field base and nx * w): 256-bit accesses
};

// 32-byte (256-bit) global accesses, sm_100: LDG.E.ENL2.256 / STG.E.ENL2.256
__device__ __forceinline__ void ld32B(const double *p, double (&v)[4]) {
    asm volatile("ld.global.nc.v4.f64 {%0, %1, %2, %3}, [%4];" : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(p));
}
__device__ __forceinline__ void ld32B(const float *p, float (&v)[8]) {
    asm volatile("ld.global.nc.v8.f32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                 : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
                 : "l"(p));
}
__device__ __forceinline__ void st32B_cs(double *p, const double (&v)[4]) {
    asm volatile("st.global.cs.v4.f64 [%0], {%1, %2, %3, %4};" ::"l"(p), "d"(v[0]), "d"(v[1]), "d"(v[2]), "d"(v[3])
                 : "memory");
}
__device__ __forceinline__ void st32B_cs(float *p, const float (&v)[8]) {
    asm volatile("st.global.cs.v8.f32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(p), "f"(v[0]), "f"(v[1]),
                 "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7])
                 : "memory");
}

template <int NDIM>
struct BlockShape;
template <>
struct BlockShape<2> {
    static constexpr int BX = 8, BY = 8, BZ = 1;
};
template <>
struct BlockShape<3> {
    static constexpr int BX = 4, BY = 4, BZ = 4;
};

// Lorenzo prediction of in-block value i from its lower neighbours (block-local:
// neighbours outside the block are 0), "3 and 7 adjacent data points".
template <int NDIM>
__device__ __forceinline__ int lorenzo_pred(const int (&q)[LND], int i) {
    using S = BlockShape<NDIM>;
    const int ix = i % S::BX, iy = (i / S::BX) % S::BY, iz = i / (S::BX * S::BY);
    auto Q = [&](int dx, int dy, int dz) -> int {
        if (ix < dx || iy < dy || iz < dz) return 0;
        return q[i - dx - dy * S::BX - dz * S::BX * S::BY];
    };
    if (NDIM == 2) return Q(1, 0, 0) + Q(0, 1, 0) - Q(1, 1, 0);
    return Q(1, 0, 0) + Q(0, 1, 0) + Q(0, 0, 1) - Q(1, 1, 0) - Q(1, 0, 1) - Q(0, 1, 1) + Q(1, 1, 1);
}

// origin (x0, y0, z0) of block b in the field
struct BlockOrigin {
    uint64_t x0, y0, z0;
};
template <int NDIM>
__device__ __forceinline__ BlockOrigin block_origin(const GeomND &g, uint64_t b) {
    using S = BlockShape<NDIM>;
    BlockOrigin o;
    const uint64_t cbx = b % g.nbx, r = b / g.nbx;
    o.x0 = cbx * S::BX;
    o.y0 = (r % g.nby) * S::BY;
    o.z0 = (r / g.nby) * S::BZ;
    return o;
}
// field linear index of in-block value i (compile-time after unrolling), or ~0
// outside the field
template <int NDIM>
__device__ __forceinline__ uint64_t nd_index(const GeomND &g, const BlockOrigin &o, int i) {
    using S = BlockShape<NDIM>;
    const int ix = i % S::BX, iy = (i / S::BX) % S::BY, iz = i / (S::BX * S::BY);
    const uint64_t x = o.x0 + ix, y = o.y0 + iy, z = o.z0 + iz;
    if (x >= g.nx || y >= g.ny || z >= g.nz) return ~uint64_t(0);
    return (z * g.ny + y) * g.nx + x;
}

// 16-byte vectors of the value type (rows of a block are 4 or 8 contiguous values)
template <typename T>
struct Vec16;
template <>
struct Vec16<float> {
    using type = float4;
    static constexpr int V = 4;
};
template <>
struct Vec16<double> {
    using type = double2;
    static constexpr int V = 2;
};

// true if block b lies entirely inside the field and its rows are 16-byte aligned
// (x extent a multiple of the vector width; the base is 16-byte aligned by the ABI)
template <typename T, int NDIM>
__device__ __forceinline__ bool interior_vec(const GeomND &g, const BlockOrigin &o) {
    using S = BlockShape<NDIM>;
    return (g.nx % Vec16<T>::V) == 0 && o.x0 + S::BX <= g.nx && o.y0 + S::BY <= g.ny &&
           o.z0 + S::BZ <= g.nz;
}

// ❶ for one value, as a BIASED pattern (f32: q + 0x4B400000 mod 2^32; f64: q).
// UNCHECKED (f32 only): the bits of fl(x·inv + 1.5·2^23), exact whenever the block passes
// the certificate in compress_nd_kernel; CHECKED: FORMAT.md §7's range check (|d| <=
// 2^ndim · max|q| must fit the 31-bit code: |x/2eb| <= 2^28-1 in 2D, 2^27-1 in 3D).
template <int NDIM, bool CHECKED>
__device__ __forceinline__ uint32_t qpattern(float x, float inv, bool &bad) {
    const float t = __fmul_rn(x, inv);
    if (!CHECKED) return static_cast<uint32_t>(__float_as_int(__fadd_rn(t, 12582912.0f)));
    bad |= !(fabsf(t) <= (NDIM == 2 ? 268435440.0f : 134217720.0f));
    return static_cast<uint32_t>(__float2int_rn(t)) + 0x4B400000u;
}
template <int NDIM, bool CHECKED>
__device__ __forceinline__ uint32_t qpattern(double x, double inv, bool &bad) {
    const double t = __dmul_rn(x, inv);
    bad |= !(fabs(t) <= (NDIM == 2 ? 268435455.0 : 134217727.0));
    return static_cast<uint32_t>(__double_as_longlong(__dadd_rn(t, 6755399441055744.0)));  // rint(t), |t| < 2^31
}

// Gather + ❶ of the 64 values of block origin bo, row by row (3D: 16 rows of 4, 2D: 8
// rows of 8 values), each row from base + roff[r] (host-computed byte offsets). Interior
// blocks of fields whose rows are whole 16-byte vectors load unpredicated vectors; edge
// blocks the same vectors predicated on lying inside the field; other fields (nx not a
// multiple of the vector width) value by value. Values outside the field (and every
// value of an inactive block) get the pattern of q = 0 and bit i of *outside.
template <typename T, int NDIM, bool CHECKED>
__device__ __forceinline__ void gather_block(const T *__restrict__ in, const GeomND &g, uint32_t x0, uint32_t y0,
                                             uint32_t z0, bool active, T inv, uint32_t (&v)[LND],
                                             uint64_t &outside, bool &bad) {
    using S = BlockShape<NDIM>;
    using VT = typename Vec16<T>::type;
    constexpr int V = Vec16<T>::V;
    constexpr int NROW = LND / S::BX;
    const char *base =
        reinterpret_cast<const char *>(in) + ((static_cast<uint64_t>(z0) * g.ny + y0) * g.nx + x0) * sizeof(T);
    uint64_t outb = 0;
    if (g.vec) {
        const bool interior = active && x0 + S::BX <= g.nx && y0 + S::BY <= g.ny && z0 + S::BZ <= g.nz;
        constexpr bool ROW32 = (S::BX * sizeof(T)) % 32 == 0;  // rows of whole 32-byte vectors
        if (interior && ROW32 && g.vec32) {
            // 256-bit loads (3D f64: one per row; 2D: two per row of 8 values)
            constexpr int V32 = 32 / sizeof(T);
            const char *rp = base;
#pragma unroll
            for (int r = 0; r < NROW; r++) {
                if (sizeof(T) == 8 && r && (r * S::BX) % 16 == 0) asm volatile("" ::: "memory");
                if (r) rp += (r % S::BY) ? g.ystep : g.zstep;
#pragma unroll
                for (int u = 0; u < S::BX / V32; u++) {
                    T tmp[V32];
                    ld32B(reinterpret_cast<const T *>(rp) + u * V32, tmp);
#pragma unroll
                    for (int k = 0; k < V32; k++) v[r * S::BX + u * V32 + k] = qpattern<NDIM, CHECKED>(tmp[k], inv, bad);
                }
            }
        } else if (interior) {
            // rows by a chain of pointer steps (so that the 16 row addresses are never
            // all live at once: 64 values + 32 address registers would spill)
            const char *rp = base;
#pragma unroll
            for (int r = 0; r < NROW; r++) {
                // f64: at most 32 loaded registers in flight (all 128 would spill)
                if (sizeof(T) == 8 && r && (r * S::BX) % 16 == 0) asm volatile("" ::: "memory");
                if (r) rp += (r % S::BY) ? g.ystep : g.zstep;
                const VT *row = reinterpret_cast<const VT *>(rp);
#pragma unroll
                for (int u = 0; u < S::BX / V; u++) {
                    T tmp[V];
                    *reinterpret_cast<VT *>(tmp) = __ldg(row + u);
#pragma unroll
                    for (int k = 0; k < V; k++) v[r * S::BX + u * V + k] = qpattern<NDIM, CHECKED>(tmp[k], inv, bad);
                }
            }
        } else {
#pragma unroll
            for (int r = 0; r < NROW; r++) {
                if (sizeof(T) == 8 && r && (r * S::BX) % 16 == 0) asm volatile("" ::: "memory");
                const uint32_t dy = r % S::BY, dz = r / S::BY;
                const bool row_ok = active && y0 + dy < g.ny && z0 + dz < g.nz;
                const VT *row = reinterpret_cast<const VT *>(base + g.roff[r]);
#pragma unroll
                for (int u = 0; u < S::BX / V; u++) {
                    const bool ok = row_ok && x0 + u * V < g.nx;  // nx % V == 0: whole vectors
                    T tmp[V];
#pragma unroll
                    for (int k = 0; k < V; k++) tmp[k] = T(0);
                    if (ok) *reinterpret_cast<VT *>(tmp) = __ldg(row + u);
                    outb |= static_cast<uint64_t>(ok ? 0u : (1u << V) - 1u) << (r * S::BX + u * V);
#pragma unroll
                    for (int k = 0; k < V; k++) v[r * S::BX + u * V + k] = qpattern<NDIM, CHECKED>(tmp[k], inv, bad);
                }
            }
        }
    } else {
#pragma unroll
        for (int r = 0; r < NROW; r++) {
            if (r && (r * S::BX) % 16 == 0) asm volatile("" ::: "memory");
            const uint32_t dy = r % S::BY, dz = r / S::BY;
            const bool row_ok = active && y0 + dy < g.ny && z0 + dz < g.nz;
            const T *row = reinterpret_cast<const T *>(base + g.roff[r]);
#pragma unroll
            for (int ix = 0; ix < S::BX; ix++) {
                const bool ok = row_ok && x0 + ix < g.nx;
                const T val = ok ? row[ix] : T(0);
                outb |= static_cast<uint64_t>(!ok) << (r * S::BX + ix);
                v[r * S::BX + ix] = qpattern<NDIM, CHECKED>(val, inv, bad);
            }
        }
    }
    outside = outb;
}

// nD Lorenzo residuals of the biased patterns, in place: the separable product of first
// differences along x, y (and z) with in-block zero boundaries, which expands to q - pred
// with FORMAT.md §7's 3- / 7-neighbour prediction ((1-S_x)(1-S_y)(1-S_z) q). The biases
// cancel in every difference except at the block's corner (value 0, no neighbour).
// Cost per 64 values: 112 (2D) / 144 (3D) integer subtractions.
template <typename T, int NDIM>
__device__ __forceinline__ void lorenzo_block(uint32_t (&v)[LND]) {
    using S = BlockShape<NDIM>;
    constexpr int NROW = LND / S::BX;
#pragma unroll
    for (int r = 0; r < NROW; r++)
#pragma unroll
        for (int ix = S::BX - 1; ix >= 1; ix--) v[r * S::BX + ix] -= v[r * S::BX + ix - 1];
#pragma unroll
    for (int z = 0; z < S::BZ; z++)
#pragma unroll
        for (int iy = S::BY - 1; iy >= 1; iy--)
#pragma unroll
            for (int ix = 0; ix < S::BX; ix++)
                v[(z * S::BY + iy) * S::BX + ix] -= v[(z * S::BY + iy - 1) * S::BX + ix];
    if (NDIM == 3) {
#pragma unroll
        for (int z = S::BZ - 1; z >= 1; z--)
#pragma unroll
            for (int m = 0; m < S::BX * S::BY; m++) v[z * S::BX * S::BY + m] -= v[(z - 1) * S::BX * S::BY + m];
    }
    v[0] -= static_cast<uint32_t>(QBias<T>::value);
}
// f32 certificate for the unchecked patterns: a block whose residuals all have |d| < 2^15
// has |q| <= 64 (2^15 - 1) < 2^22 everywhere (q is the in-block box sum of at most 64
// residuals, modulo 2^32 as computed), so every pattern lies strictly inside the binade
// where the RN addition is rint(t) exactly and |t| < 2^22 passes the range check (the 1D
// kernel's argument, quantize_block_unchecked); NaN and ±Inf fall outside it.
constexpr int ND_FAST_FL_MAX = 15;

// One block's nD payload (FORMAT.md §7: sign 8 B, nob outlier bytes, then planes
// k = 0..fl-1 as (lo word, hi word)) to smem at byte `st` (any alignment). With the
// plane region at ps = st + 8 + nob, r = ps & 3 and P_k the k-th plane word
// (P_2j = lo[j], P_2j+1 = hi[j]; P_-1, P_-2, P_-3 the header words ending at ps), the
// aligned word at ps - r + 4k is funnel(P_k-1, P_k, 8r): every aligned word that lies
// inside the payload is one 32-bit store; the <= 3 head bytes and <= 3 tail bytes, whose
// words the neighbouring blocks share, are byte stores. No atomics and no pre-zeroed
// memory (each byte of the ring has exactly one writer).
template <int R>
__device__ __forceinline__ void stage_payload_nd(uint8_t *base, uint32_t st, uint64_t sign, uint32_t outl, int nob,
                                                 int fl, const uint32_t (&lo)[32], const uint32_t (&hi)[32]) {
    const uint32_t h0 = static_cast<uint32_t>(sign), h1 = static_cast<uint32_t>(sign >> 32), h2 = outl;
    const uint32_t ps = st + 8u + nob;
    const uint32_t r = ps & 3u;
    const uint32_t sh = 8u * r;
    uint32_t *w = reinterpret_cast<uint32_t *>(base + ps - r);
    const uint32_t pm1 = static_cast<uint32_t>(((static_cast<uint64_t>(h2) << 32) | h1) >> (8 * nob));  // [4+nob, 8+nob)
    const uint32_t pm2 = static_cast<uint32_t>(sign >> (8 * nob));                                   // [nob, nob+4)
    const uint32_t pm3 = static_cast<uint32_t>(static_cast<uint64_t>(h0) << (32 - 8 * nob));  // top nob bytes
    w[-1] = __funnelshift_l(pm2, pm1, sh);  // payload bytes [4 + nob - r, 8 + nob - r): always inside
    if (static_cast<uint32_t>(nob) >= r) w[-2] = __funnelshift_l(pm3, pm2, sh);
    if (nob == 4 && r == 0) w[-3] = h0;
    // head bytes [0, hb): the payload bytes before the first word written above
    const uint32_t hb = (nob == 4 && r == 0) ? 0u : (static_cast<uint32_t>(nob) >= r ? nob - r : 4u + nob - r);
#pragma unroll
    for (uint32_t i = 0; i < 3; i++)
        if (i < hb) base[st + i] = static_cast<uint8_t>(h0 >> (8 * i));
    uint32_t prev = pm1;
#pragma unroll
    for (int j = 0; j < R; j++) {
        if (j < fl) {
            w[2 * j] = __funnelshift_l(prev, lo[j], sh);
            w[2 * j + 1] = __funnelshift_l(lo[j], hi[j], sh);
            prev = hi[j];
        }
    }
    // tail bytes: the last r payload bytes (the top r bytes of the last word)
    uint8_t *tb = base + ps - r + 8u * fl;
#pragma unroll
    for (uint32_t i = 0; i < 3; i++)
        if (i < r) tb[i] = static_cast<uint8_t>(prev >> (8 * (4 - r + i)));
}

constexpr uint32_t ND_STAGE = BPT * 4 * LND + 64;  // max tile payload + slack (decompression)
constexpr uint32_t ND_TILE_MAX = BPT * 4 * LND;      // largest tile payload (Plain, fl = 31)
constexpr uint32_t ND_RING = 96 * 1024;              // compression staging ring (>= ND_TILE_MAX)

// Warp-specialised persistent compression CTAs (NT_COMP = 288 threads: 8 producer warps,
// one thread per 64-value block, + 1 resolver warp; 2 CTAs per SM), the same structure
// as the 1D compress_kernel: producer thread 0 claims tiles in order from an atomic
// ticket (after staging the previous one, so a claimed tile never waits on a lookback
// before it publishes) and hands the ticket over through an mbarrier; the producers
// gather their blocks straight from global memory (16-byte rows for interior blocks),
// encode, scan (one named barrier), publish the aggregate, stage the payload in the
// shared byte ring (byte-exact, no clearing) and queue the tile; the resolver warp runs
// each queued tile's decoupled lookback and copies its payload out, in order. No CTA-wide
// barrier waits on a lookback (round 1 ran it in warp 0 between two __syncthreads).
constexpr uint32_t ND_RING_V = 128 * 1024;  // virtual lap of the ring (a power of 2 >= ND_RING)

template <typename T, int NDIM, bool OUTLIER, int LBR = LB_PER_LANE>
__global__ void __launch_bounds__(NT_COMP, 2) compress_nd_kernel(const T *__restrict__ in, const GeomND g,
                                                                 const double eb_abs_arg,
                                                                 const int eb_from_header,
                                                                 uint8_t *__restrict__ out,
                                                                 unsigned *__restrict__ ticket,
                                                                 uint64_t *__restrict__ d_out_bytes,
                                                                 const HdrStatic hs) {
    extern __shared__ uint8_t stage_raw[];
    uint8_t *ring = smem_align<16>(stage_raw);
    __shared__ uint64_t s_full;                    // thread 0 -> producers: the claimed ticket
    __shared__ uint64_t s_staged[NQ], s_done[NQ];  // queue slots: producers -> resolver -> producers
    __shared__ uint64_t s_qt[NQ];
    __shared__ uint32_t s_qagg[NQ], s_qpos[NQ];
    __shared__ uint8_t s_qbad[NQ];
    __shared__ uint32_t s_warp[2][NT / 32];  // tile_scan_1bar, by tile parity
    __shared__ uint32_t s_tailb[2];          // s_tail as thread 0 acquired it before the scan, by parity
    __shared__ uint32_t s_tail;              // ring bytes released by the resolver
    __shared__ uint32_t s_tkin;
    __shared__ volatile uint32_t s_end;  // queue index of the end marker
    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const uint64_t T_eff = g.T ? g.T : 1;
    uint64_t *index = reinterpret_cast<uint64_t *>(out + 64);
    const double eb_abs =
        eb_from_header ? *reinterpret_cast<const volatile double *>(out + 32) : eb_abs_arg;

    if (tid == 0) {
        s_end = 0xFFFFFFFFu;
        s_tail = 0;
        mbar_init(&s_full, 1);
        for (int i = 0; i < NQ; i++) {
            mbar_init(&s_staged[i], NT / 32);
            mbar_init(&s_done[i], 1);
        }
        fence_mbar_init();
        s_tkin = atomicAdd(ticket, 1u);  // in-order tiles: forward progress
        mbar_arrive(&s_full);
    }
    __syncthreads();

    if (warp < RESOLVE_WARP) {
        // ============================== producers
        const auto K = make_consts(eb_abs, static_cast<T *>(nullptr));
        uint32_t head = 0;  // ring allocation cursor, identical in every producer thread
        for (uint32_t it = 0;; ++it) {
            const int qs = it % NQ;
            if (tid == 0) s_tailb[it & 1] = ld_acquire_cta(&s_tail);  // handed over by the scan barrier
            mbar_wait(&s_full, it & 1);
            const uint64_t t = s_tkin;
            if (t >= T_eff) {  // end marker for the resolver (one arrival per warp)
                if (lane == 0) {
                    if (it >= NQ) mbar_wait(&s_done[qs], (it / NQ - 1) & 1);
                    if (tid == 0) s_end = it;
                    mbar_arrive(&s_staged[qs]);
                }
                break;
            }
            const uint64_t b = t * BPT + tid;
            const bool active = b < g.nb;
            uint32_t x0, y0, z0;  // block origin (every extent is < 2^32)
            {
                using S = BlockShape<NDIM>;
                const uint64_t bb = active ? b : 0;
                uint32_t cbx, cby, cbz;
                if (g.nb < (1ull << 31)) {
                    const uint32_t r32 = fast_div(static_cast<uint32_t>(bb), g.dbx);
                    const uint32_t z32 = fast_div(r32, g.dby);
                    cbx = static_cast<uint32_t>(bb) - r32 * static_cast<uint32_t>(g.nbx);
                    cby = r32 - z32 * static_cast<uint32_t>(g.nby);
                    cbz = z32;
                } else {
                    const uint64_t r = bb / g.nbx, z = r / g.nby;
                    cbx = static_cast<uint32_t>(bb - r * g.nbx);
                    cby = static_cast<uint32_t>(r - z * g.nby);
                    cbz = static_cast<uint32_t>(z);
                }
                x0 = cbx * S::BX;
                y0 = cby * S::BY;
                z0 = cbz * S::BZ;
            }
            // ---- gather + ❶ (f32: unchecked patterns, redone checked if the block fails the
            //      certificate) + nD Lorenzo residuals
            uint32_t v[LND];
            uint64_t outside;
            bool bad = false;
            uint32_t(&a)[LND] = v;  // residual magnitudes, in place
            uint32_t sign_lo = 0, sign_hi = 0, or_rest = 0;
            auto residuals = [&]() {
                lorenzo_block<T, NDIM>(v);
                if (outside) {  // values outside the field have residual 0 (FORMAT.md §7)
#pragma unroll
                    for (int i = 0; i < LND; i++)
                        if ((outside >> i) & 1ull) v[i] = 0;
                }
                or_rest = 0;
#pragma unroll
                for (int i = LND - 1; i >= 0; i--) {
                    const int d = static_cast<int>(v[i]);
                    a[i] = static_cast<uint32_t>(d < 0 ? -d : d);
                    if (i >= 32)
                        sign_hi = __funnelshift_l(static_cast<uint32_t>(d), sign_hi, 1);  // bit i-32 = d_i < 0
                    else
                        sign_lo = __funnelshift_l(static_cast<uint32_t>(d), sign_lo, 1);
                    if (i) or_rest |= a[i];
                }
            };
            if (sizeof(T) == 4) {
                gather_block<T, NDIM, false>(in, g, x0, y0, z0, active, K.inv, v, outside, bad);
                residuals();
                if (32 - __clz(or_rest | a[0]) > ND_FAST_FL_MAX) {
                    gather_block<T, NDIM, true>(in, g, x0, y0, z0, active, K.inv, v, outside, bad);
                    residuals();
                }
            } else {
                gather_block<T, NDIM, true>(in, g, x0, y0, z0, active, K.inv, v, outside, bad);
                residuals();
            }
            const uint64_t sign = static_cast<uint64_t>(sign_lo) | (static_cast<uint64_t>(sign_hi) << 32);
            // ---- ❷ FLE with 8-byte fields
            const int fl_p = 32 - __clz(or_rest | a[0]);
            uint32_t size = fl_p ? 8u * (1u + fl_p) : 0u;
            uint32_t obyte = static_cast<uint32_t>(fl_p);
            int fl = fl_p, nob = 0;
            if (OUTLIER) {
                const int fl_o = 32 - __clz(or_rest);
                const int ob = max(1, (32 - __clz(a[0]) + 7) >> 3);
                const uint32_t size_o = 8u + ob + 8u * fl_o;
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

            // ---- ❸ intra-tile scan (one barrier among the producers, with the range
            //      flag); publish the aggregate at once
            uint32_t agg;
            bool any_bad;
            const uint32_t my_excl = tile_scan_1bar(size, bad, s_warp[it & 1], &agg, &any_bad, BAR_PROD);
            if (tid == 0 && g.T) publish_aggregate(index, t, agg, any_bad);
            if (active) out[g.O + b] = static_cast<uint8_t>(obyte);

            // ---- ring room (16-aligned region, no lap straddle); the cursor thread 0
            //      acquired before the barrier, else spin with acquire loads
            uint32_t pos = (head + 15u) & ~15u;
            if ((pos % ND_RING_V) + agg > ND_RING) pos = (pos / ND_RING_V + 1) * ND_RING_V;
            auto fits = [&](uint32_t tl) { return pos + agg <= tl + ND_RING_V || tl == head; };
            if (!fits(s_tailb[it & 1]))
                while (!fits(ld_acquire_cta(&s_tail))) __nanosleep(64);
            head = pos + agg;

            // ---- payload into the ring: sign (8 B), outlier (nob B), planes (8 B each:
            //      values 0..31 then 32..63), bit planes by two in-register transposes
            const uint32_t outl = a[0];
            if (OUTLIER && nob) a[0] = 0;
            uint32_t(&lo)[32] = *reinterpret_cast<uint32_t(*)[32]>(&a[0]);   // values 0..31
            uint32_t(&hi)[32] = *reinterpret_cast<uint32_t(*)[32]>(&a[32]);  // values 32..63
            const int flw = static_cast<int>(__reduce_max_sync(0xffffffffu, static_cast<unsigned>(size ? fl : 0)));
            uint8_t *stg = ring + (pos % ND_RING_V);
            if (flw == 0) {
                if (size) stage_payload_nd<0>(stg, my_excl, sign, outl, nob, 0, lo, hi);
            } else if (flw <= 1) {
                pack_planes<0>(lo);
                pack_planes<0>(hi);
                if (size) stage_payload_nd<1>(stg, my_excl, sign, outl, nob, fl, lo, hi);
            } else if (flw <= 2) {
                pack_planes<1>(lo);
                pack_planes<1>(hi);
                if (size) stage_payload_nd<2>(stg, my_excl, sign, outl, nob, fl, lo, hi);
            } else if (flw <= 4) {
                pack_planes<2>(lo);
                pack_planes<2>(hi);
                if (size) stage_payload_nd<4>(stg, my_excl, sign, outl, nob, fl, lo, hi);
            } else if (flw <= 8) {
                pack_planes<3>(lo);
                pack_planes<3>(hi);
                if (size) stage_payload_nd<8>(stg, my_excl, sign, outl, nob, fl, lo, hi);
            } else if (flw <= 16) {
                pack_planes<4>(lo);
                pack_planes<4>(hi);
                if (size) stage_payload_nd<16>(stg, my_excl, sign, outl, nob, fl, lo, hi);
            } else {
                pack_planes<5>(lo);
                pack_planes<5>(hi);
                if (size) stage_payload_nd<32>(stg, my_excl, sign, outl, nob, fl, lo, hi);
            }

            // ---- queue the tile (one arrival per warp; thread 0 fills in the slot)
            __syncwarp();
            if (lane == 0) {
                if (it >= NQ) mbar_wait(&s_done[qs], (it / NQ - 1) & 1);  // queue slot free
                if (tid == 0) {
                    s_qt[qs] = t;
                    s_qagg[qs] = agg;
                    s_qbad[qs] = any_bad;
                    s_qpos[qs] = pos;
                }
                mbar_arrive(&s_staged[qs]);
            }
            // ---- claim the next tile (nothing unpublished is held now)
            if (tid == 0) {
                s_tkin = atomicAdd(ticket, 1u);
                mbar_arrive(&s_full);
            }
        }
    } else {
        // ============================== resolver: ❸ then ❹, in tile order
        for (uint32_t it = 0;; ++it) {
            const int q = it % NQ;
            mbar_wait_backoff(&s_staged[q], (it / NQ) & 1, 100);
            if (it >= s_end) break;
            const uint64_t t = s_qt[q];
            const uint32_t agg = s_qagg[q];
            const uint32_t pos = s_qpos[q];
            const bool bad = s_qbad[q];
            bool rng = bad;
            uint64_t excl = 0;
            if (g.T && t > 0) excl = lookback<LBR>(index, t, agg, bad, &rng);
            const uint64_t dst0 = g.D + excl;
            write_payload(ring + (pos % ND_RING_V), out, dst0, agg, lane, 32);
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
                    h[1] = hs.eb_mode | (status << 8) | (static_cast<uint64_t>(BPT) << 16) |
                           (static_cast<uint64_t>(NDIM - 1) << 32);
                    h[2] = g.n;
                    h[3] = static_cast<uint64_t>(__double_as_longlong(hs.eb_user));
                    h[4] = static_cast<uint64_t>(__double_as_longlong(eb_abs));
                    h[5] = pb;
                    h[6] = total;
                    h[7] = g.nx | (g.ny << 32);
                    if (d_out_bytes) *d_out_bytes = total;
                }
            }
            __syncwarp();  // every lane's reads of these ring bytes are ordered before the release
            if (lane == 0) {
                __threadfence_block();  // release pattern: fence, then the relaxed cursor store
                st_relaxed_cta(&s_tail, pos + agg);  // in order, so the ring frees in order
                mbar_arrive(&s_done[q]);
            }
        }
    }
}

// Inverse of lorenzo_block: in-block prefix sums along x, y (and z) of the residuals
// (mod 2^32), i.e. q = box sum of d — the separable form of q_i = d_i + pred_i in index
// order (FORMAT.md §7); 112 (2D) / 144 (3D) integer additions per block. The last
// direction's sums run row by row and each finished row is handed to emit(r) at once, so
// that the stores spread over the arithmetic instead of leaving in one burst.
template <int NDIM, typename Emit>
__device__ __forceinline__ void inv_lorenzo_block(uint32_t (&v)[LND], Emit &&emit) {
    using S = BlockShape<NDIM>;
    constexpr int NROW = LND / S::BX;
#pragma unroll
    for (int r = 0; r < NROW; r++)
#pragma unroll
        for (int ix = 1; ix < S::BX; ix++) v[r * S::BX + ix] += v[r * S::BX + ix - 1];
    if (NDIM == 2) {
#pragma unroll
        for (int iy = 0; iy < S::BY; iy++) {
            if (iy)
#pragma unroll
                for (int ix = 0; ix < S::BX; ix++) v[iy * S::BX + ix] += v[(iy - 1) * S::BX + ix];
            emit(iy);
        }
    } else {
#pragma unroll
        for (int z = 0; z < S::BZ; z++)
#pragma unroll
            for (int iy = 1; iy < S::BY; iy++)
#pragma unroll
                for (int ix = 0; ix < S::BX; ix++)
                    v[(z * S::BY + iy) * S::BX + ix] += v[(z * S::BY + iy - 1) * S::BX + ix];
#pragma unroll
        for (int z = 0; z < S::BZ; z++) {
            if (z)
#pragma unroll
                for (int m = 0; m < S::BX * S::BY; m++) v[z * S::BX * S::BY + m] += v[(z - 1) * S::BX * S::BY + m];
#pragma unroll
            for (int iy = 0; iy < S::BY; iy++) emit(z * S::BY + iy);
        }
    }
}

constexpr uint32_t ND_DRING = 96 * 1024;  // decompression payload ring per CTA (2 x 64 KiB + 16 do not fit:
                                         // the next payload goes behind the current one or waits)

// Persistent decompression CTAs (256 threads, one per 64-value block; 2 per SM): CTA c
// decodes tiles c, c + G, ...; each tile's payload range comes from the persisted tile
// index in O(1) (R-14) and is bulk-loaded (1D TMA) into a 96 KiB ring while the previous
// tile is decoded (the 1D decompress_kernel's scheme: behind the current payload, else
// at the ring's start, else deferred until the ring is empty); index words and offset
// bytes are fetched two tiles ahead. Per block: scan of the 256 sizes, sign / outlier /
// two 32x32 plane transposes (values 0..31, 32..63), prefix sums (inverse Lorenzo),
// I2FP + FMUL, 16-byte streaming row stores (edge blocks value by value, bounds-checked).
template <typename T, int NDIM>
__global__ void __launch_bounds__(NT, 2) decompress_nd_kernel(const uint8_t *__restrict__ cmp, T *__restrict__ out,
                                                           const GeomND g, int *__restrict__ d_status) {
    extern __shared__ uint8_t stage_raw[];
    uint8_t *ring = smem_align<16>(stage_raw);
    __shared__ uint64_t s_bar[2];
    __shared__ uint32_t s_warp[2][NT / 32];  // the scan's warp totals, by tile parity
    __shared__ uint64_t s_excl[2];
    __shared__ uint32_t s_bytes[2];
    __shared__ uint32_t s_rpos[2];
    __shared__ double s_eb;
    __shared__ int s_err;
    using S = BlockShape<NDIM>;
    const int tid = threadIdx.x;
    const uint64_t G = gridDim.x;
    const uint64_t *index = reinterpret_cast<const uint64_t *>(cmp) + 8;
    constexpr uint32_t BAD_BYTES = 0xFFFFFFFFu;
    uint64_t raw_p = FLAG_P, raw_i = 0, pb_hdr = 0;
    bool pending = false, deferred = false;
    uint32_t r_pos = 0, r_len = 0;
    auto launch = [&](uint64_t dp, uint64_t di, int bi, bool ring_empty) -> bool {
        const uint64_t e = dp & VAL_MASK, i = di & VAL_MASK;
        uint32_t bytes = BAD_BYTES;
        if ((dp >> 61) == 4 && (di >> 61) == 4 && i >= e && i <= pb_hdr && i - e <= static_cast<uint64_t>(BPT) * 4 * LND)
            bytes = static_cast<uint32_t>(i - e);
        s_excl[bi] = e;
        s_bytes[bi] = bytes;
        if (bytes != BAD_BYTES && bytes) {
            const uint64_t src0 = (g.D + e) & ~uint64_t(15);
            const uint32_t len = static_cast<uint32_t>(roundup16(g.D + e + bytes) - src0);
            uint32_t pos;
            if (ring_empty)
                pos = 0;
            else if (r_pos + r_len + len <= ND_DRING - 16)
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
        const uint64_t *h = reinterpret_cast<const uint64_t *>(cmp);
        const uint64_t h0 = h[0], h1 = h[1];
        int err = 0;
        const uint32_t want1 = 1u | (static_cast<uint32_t>(Traits<T>::DTYPE) << 8) | (6u << 24);
        if ((h0 & 0xFFFFFFFFu) != MAGIC || ((h0 >> 32) & 0xFF00FFFFu) != want1 ||
            ((h1 >> 16) & 0xFFFFu) != BPT || ((h1 >> 32) & 0xFFu) != static_cast<uint64_t>(NDIM - 1) ||
            h[2] != g.n || h[7] != (g.nx | (g.ny << 32)))
            err = ST_FORMAT;
        else if (((h1 >> 8) & 0xFF) != 0)
            err = ((h1 >> 8) & 0xFF) == ST_RANGE ? ST_RANGE : ST_FORMAT;
        pb_hdr = h[5];
        if (!err && h[6] != roundup16(g.D + pb_hdr)) err = ST_FORMAT;
        s_err = err;
        s_eb = __longlong_as_double(static_cast<long long>(h[4]));
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
    // block payload size and reserved-bit check from an offset byte (FORMAT.md §4)
    auto bsize = [](uint32_t ob, bool &bad) {
        const uint32_t f = ob & 31u;
        const bool o = (ob & 0x80u) != 0;
        bad = !o && (ob & 0x60u);
        return o ? 8u + (((ob >> 5) & 3u) + 1u) + 8u * f : (f ? 8u * (1u + f) : 0u);
    };
    // The scan of a tile's 256 block sizes is computed one tile ahead (its offset bytes
    // are prefetched), its warp totals crossing the CTA barrier that the current tile
    // needs anyway: one barrier per tile instead of two.
    uint32_t my_excl, agg;
    bool any_bad;
    {
        bool bd;
        const uint32_t sz = bsize(ob_cur, bd);
        const uint32_t inc = scan_part1(sz, bd, s_warp[0]);
        __syncthreads();
        my_excl = scan_part2(sz, inc, s_warp[0], &agg, &any_bad);
    }
    int err = 0;
    for (uint32_t it = 0; t < g.T; ++it, t += G) {
        const int cur = it & 1;
        const uint64_t tn = t + G;
        uint64_t nraw_p = 0, nraw_i = 0;
        if (tid == 0) {
            pending = false;
            deferred = false;
            if (tn < g.T) {  // the next tile's payload streams in during this one
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
        uint32_t ob_pref = 0;  // offset byte of tile t + 2G
        {
            const uint64_t t2 = tn + G;
            const uint64_t b2 = t2 * BPT + tid;
            if (t2 < g.T && b2 < g.nb) ob_pref = cmp[g.O + b2];
        }
        const uint64_t b = t * BPT + tid;
        const bool active = b < g.nb;
        const uint32_t obyte = ob_cur;
        const uint32_t fl = obyte & 31u;
        const bool is_o = (obyte & 0x80u) != 0;
        const uint32_t nob = is_o ? ((obyte >> 5) & 3u) + 1u : 0u;
        const bool bad = (!is_o && (obyte & 0x60u));
        const uint32_t size = is_o ? 8u + nob + 8u * fl : (fl ? 8u * (1u + fl) : 0u);
        (void)bad;
        // the payload's arrival also orders thread 0's s_bytes / s_excl / s_rpos writes for
        // this tile (its expect_tx arrival releases them), even when they were made after
        // the last barrier (a deferred launch)
        mbar_wait(&s_bar[cur], (it >> 1) & 1);
        if (any_bad || agg != s_bytes[cur]) {
            err = ST_FORMAT;
            if (tid == 0 && pending) mbar_wait(&s_bar[cur ^ 1], ((it + 1) >> 1) & 1);
            break;
        }

        // ---- ❷⁻¹: sign (8 B), outlier, planes (8 B each) -> residual magnitudes
        uint32_t v[LND];
        uint32_t(&lo)[32] = *reinterpret_cast<uint32_t(*)[32]>(&v[0]);
        uint32_t(&hi)[32] = *reinterpret_cast<uint32_t(*)[32]>(&v[32]);
        uint32_t sign_lo = 0, sign_hi = 0, outl = 0;
        const int flw = static_cast<int>(__reduce_max_sync(0xffffffffu, size ? fl : 0u));
        {
            const uint8_t *pbuf = ring + s_rpos[cur];
            uint32_t p = static_cast<uint32_t>((g.D + s_excl[cur]) & 15u) + my_excl;
            if (size) {
                sign_lo = ld_u32_unaligned(pbuf, p);
                sign_hi = ld_u32_unaligned(pbuf, p + 4);
                p += 8;
                if (is_o) {
                    outl = ld_u32_unaligned(pbuf, p);
                    if (nob < 4) outl &= (1u << (8 * nob)) - 1u;
                    p += nob;
                }
            }
            // plane k = (lo word, hi word) at p + 8k: one funnel of two aligned words each
            const uint32_t *w = reinterpret_cast<const uint32_t *>(pbuf + (p & ~3u));
            const uint32_t sh = 8u * (p & 3u);
            auto planes = [&](auto RC) {
                constexpr int R = decltype(RC)::value;
                uint32_t prev = size ? w[0] : 0u;
#pragma unroll
                for (int k = 0; k < R; k++) {
                    uint32_t l = 0, hh = 0;
                    if (size && k < (int)fl) {
                        const uint32_t w1 = w[2 * k + 1], w2 = w[2 * k + 2];
                        l = __funnelshift_r(prev, w1, sh);
                        hh = __funnelshift_r(w1, w2, sh);
                        prev = w2;
                    }
                    lo[k] = l;
                    hi[k] = hh;
                }
#pragma unroll
                for (int k = R; k < 32; k++) lo[k] = hi[k] = 0;
            };
            if (flw == 0) {
#pragma unroll
                for (int k = 0; k < 32; k++) lo[k] = hi[k] = 0;
            } else if (flw <= 1) {
                planes(std::integral_constant<int, 1>());
                unpack_planes<0>(lo);
                unpack_planes<0>(hi);
            } else if (flw <= 2) {
                planes(std::integral_constant<int, 2>());
                unpack_planes<1>(lo);
                unpack_planes<1>(hi);
            } else if (flw <= 4) {
                planes(std::integral_constant<int, 4>());
                unpack_planes<2>(lo);
                unpack_planes<2>(hi);
            } else if (flw <= 8) {
                planes(std::integral_constant<int, 8>());
                unpack_planes<3>(lo);
                unpack_planes<3>(hi);
            } else if (flw <= 16) {
                planes(std::integral_constant<int, 16>());
                unpack_planes<4>(lo);
                unpack_planes<4>(hi);
            } else {
                planes(std::integral_constant<int, 32>());
                unpack_planes<5>(lo);
                unpack_planes<5>(hi);
            }
        }
        // the next tile's scan, part 1 (its warp totals cross the barrier below)
        bool bad_n;
        const uint32_t size_n = tn < g.T ? bsize(ob_next, bad_n) : (bad_n = false, 0u);
        const uint32_t inc_n = scan_part1(size_n, bad_n, s_warp[cur ^ 1]);
        __syncthreads();  // every thread has read this tile's payload from the ring
        if (tid == 0 && deferred) {  // the ring is empty now: fetch the next payload
            launch(nraw_p, nraw_i, cur ^ 1, true);
            pending = true;
        }
        uint32_t agg_n;
        bool any_bad_n;
        const uint32_t my_excl_n = scan_part2(size_n, inc_n, s_warp[cur ^ 1], &agg_n, &any_bad_n);
        if (is_o) lo[0] = outl;
#pragma unroll
        for (int i = 0; i < 32; i++) {
            if ((sign_lo >> i) & 1u) lo[i] = 0u - lo[i];
            if ((sign_hi >> i) & 1u) hi[i] = 0u - hi[i];
        }
        // ---- inverse Lorenzo (residuals -> q), ❶⁻¹ and the stores, row by row
        uint32_t x0 = 0, y0 = 0, z0 = 0;
        if (active) {
            uint32_t cbx, cby, cbz;
            if (g.nb < (1ull << 31)) {
                const uint32_t r32 = fast_div(static_cast<uint32_t>(b), g.dbx);
                const uint32_t z32 = fast_div(r32, g.dby);
                cbx = static_cast<uint32_t>(b) - r32 * static_cast<uint32_t>(g.nbx);
                cby = r32 - z32 * static_cast<uint32_t>(g.nby);
                cbz = z32;
            } else {
                const uint64_t r = b / g.nbx, z = r / g.nby;
                cbx = static_cast<uint32_t>(b - r * g.nbx);
                cby = static_cast<uint32_t>(r - z * g.nby);
                cbz = static_cast<uint32_t>(z);
            }
            x0 = cbx * S::BX;
            y0 = cby * S::BY;
            z0 = cbz * S::BZ;
        }
        char *base = reinterpret_cast<char *>(out) + ((static_cast<uint64_t>(z0) * g.ny + y0) * g.nx + x0) * sizeof(T);
        const bool interior = active && g.vec && x0 + S::BX <= g.nx && y0 + S::BY <= g.ny && z0 + S::BZ <= g.nz;
        char *rp = base;
        constexpr bool ROW32 = (S::BX * sizeof(T)) % 32 == 0;  // 2D f32 rows: one 256-bit store
        const bool wide = ROW32 && g.vec32;
        inv_lorenzo_block<NDIM>(v, [&](int r) {
            if (interior && wide) {
                constexpr int V32 = 32 / sizeof(T);
                if (r) rp += (r % S::BY) ? g.ystep : g.zstep;
#pragma unroll
                for (int u = 0; u < S::BX / V32; u++) {
                    T tmp[V32];
#pragma unroll
                    for (int k = 0; k < V32; k++) tmp[k] = dequantize(static_cast<int>(v[r * S::BX + u * V32 + k]), K.s);
                    st32B_cs(reinterpret_cast<T *>(rp) + u * V32, tmp);
                }
            } else if (interior) {
                using VT = typename Vec16<T>::type;
                constexpr int V = Vec16<T>::V;
                if (r) rp += (r % S::BY) ? g.ystep : g.zstep;
#pragma unroll
                for (int u = 0; u < S::BX / V; u++) {
                    T tmp[V];
#pragma unroll
                    for (int k = 0; k < V; k++) tmp[k] = dequantize(static_cast<int>(v[r * S::BX + u * V + k]), K.s);
                    __stcs(reinterpret_cast<VT *>(rp) + u, *reinterpret_cast<VT *>(tmp));
                }
            } else if (active) {
                const uint32_t dy = r % S::BY, dz = r / S::BY;
                const bool row_ok = y0 + dy < g.ny && z0 + dz < g.nz;
                T *row = reinterpret_cast<T *>(base + g.roff[r]);
#pragma unroll
                for (int ix = 0; ix < S::BX; ix++)
                    if (row_ok && x0 + ix < g.nx) row[ix] = dequantize(static_cast<int>(v[r * S::BX + ix]), K.s);
            }
        });
        ob_cur = ob_next;
        ob_next = ob_pref;
        my_excl = my_excl_n;
        agg = agg_n;
        any_bad = any_bad_n;
    }
    if (tid == 0 && err && d_status) atomicOr(d_status, err);
}

// One CTA per tile (3 per SM; grid = tiles), the round-1/2 decompressor, kept for f64:
// there its 24 warps per SM and value-order inverse Lorenzo (each value stored as soon as
// it is final) sustain the store stream better than the persistent kernel's 16 warps
// with 32 16-byte stores per thread per tile (0.266 vs 0.315 ms on config 4b, 512^3 f64;
// profiles/ab_nd_r03j.txt: long-scoreboard waits on the stores' source registers).
template <typename T, int NDIM>
__global__ void __launch_bounds__(NT, 3) decompress_nd_tile_kernel(const uint8_t *__restrict__ cmp,
                                                           T *__restrict__ out, const GeomND g,
                                                           int *__restrict__ d_status) {
    extern __shared__ uint8_t stage_raw[];
    uint8_t *pbuf = smem_align<16>(stage_raw);
    __shared__ uint64_t s_bar;
    __shared__ uint32_t s_warp[NT / 32];
    __shared__ uint64_t s_excl;
    __shared__ uint32_t s_bytes;
    __shared__ double s_eb;
    __shared__ int s_err;
    const int tid = threadIdx.x;
    const uint64_t t = blockIdx.x;
    if (tid == 0) {
        const uint64_t *h = reinterpret_cast<const uint64_t *>(cmp);
        const uint64_t h0 = h[0], h1 = h[1];
        int err = 0;
        const uint32_t want1 = 1u | (static_cast<uint32_t>(Traits<T>::DTYPE) << 8) | (6u << 24);
        if ((h0 & 0xFFFFFFFFu) != MAGIC || ((h0 >> 32) & 0xFF00FFFFu) != want1 ||
            ((h1 >> 16) & 0xFFFFu) != BPT || ((h1 >> 32) & 0xFFu) != static_cast<uint64_t>(NDIM - 1) ||
            h[2] != g.n || h[7] != (g.nx | (g.ny << 32)))
            err = ST_FORMAT;
        else if (((h1 >> 8) & 0xFF) != 0)
            err = ((h1 >> 8) & 0xFF) == ST_RANGE ? ST_RANGE : ST_FORMAT;
        const uint64_t pb = h[5];
        if (!err && h[6] != roundup16(g.D + pb)) err = ST_FORMAT;
        uint64_t e = 0, i = 0;
        if (!err && t < g.T) {
            const uint64_t *index = h + 8;
            const uint64_t dp = t ? index[t - 1] : FLAG_P, di = index[t];
            e = dp & VAL_MASK;
            i = di & VAL_MASK;
            if ((dp >> 61) != 4 || (di >> 61) != 4 || i < e || i > pb ||
                i - e > static_cast<uint64_t>(BPT) * 4 * LND)
                err = ST_FORMAT;
        }
        s_err = err;
        s_eb = __longlong_as_double(static_cast<long long>(h[4]));
        s_excl = e;
        s_bytes = static_cast<uint32_t>(i - e);
        mbar_init(&s_bar, 1);
        fence_mbar_init();
        if (!err && t < g.T) {
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
    if (s_err || t >= g.T) {
        if (tid == 0 && s_err && d_status) atomicOr(d_status, s_err);
        return;
    }
    const uint64_t b = t * BPT + tid;
    const bool active = b < g.nb;
    const uint32_t obyte = active ? cmp[g.O + b] : 0u;
    const uint32_t fl = obyte & 31u;
    const bool is_o = (obyte & 0x80u) != 0;
    const uint32_t nob = is_o ? ((obyte >> 5) & 3u) + 1u : 0u;
    bool bad = (!is_o && (obyte & 0x60u));
    const uint32_t size = is_o ? 8u + nob + 8u * fl : (fl ? 8u * (1u + fl) : 0u);
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
    // ---- ❷⁻¹: sign (8 B), outlier, planes (8 B each) -> residual magnitudes
    uint32_t lo[32], hi[32];
#pragma unroll
    for (int i = 0; i < 32; i++) lo[i] = hi[i] = 0;
    uint64_t sign = 0;
    uint32_t outl = 0;
    const int flw = static_cast<int>(__reduce_max_sync(0xffffffffu, size ? fl : 0u));
    if (size) {
        uint32_t p = static_cast<uint32_t>((g.D + s_excl) & 15u) + my_excl;
        sign = ld_u32_unaligned(pbuf, p) | (static_cast<uint64_t>(ld_u32_unaligned(pbuf, p + 4)) << 32);
        p += 8;
        if (is_o) {
            outl = ld_u32_unaligned(pbuf, p);
            if (nob < 4) outl &= (1u << (8 * nob)) - 1u;
            p += nob;
        }
#pragma unroll
        for (int k = 0; k < 32; k++) {
            if (k < (int)fl) {
                lo[k] = ld_u32_unaligned(pbuf, p + 8 * k);
                hi[k] = ld_u32_unaligned(pbuf, p + 8 * k + 4);
            }
        }
    }
    if (flw > 0) {
        if (flw <= 4) {
            unpack_planes<2>(lo);
            unpack_planes<2>(hi);
        } else if (flw <= 8) {
            unpack_planes<3>(lo);
            unpack_planes<3>(hi);
        } else if (flw <= 16) {
            unpack_planes<4>(lo);
            unpack_planes<4>(hi);
        } else {
            unpack_planes<5>(lo);
            unpack_planes<5>(hi);
        }
    }
    if (is_o) lo[0] = outl;
    // ---- inverse nD Lorenzo in index order, ❶⁻¹, scatter to the field
    int q[LND];
#pragma unroll
    for (int i = 0; i < LND; i++) {
        const uint32_t m = i < 32 ? lo[i] : hi[i - 32];
        const int d = ((sign >> i) & 1ull) ? -static_cast<int>(m) : static_cast<int>(m);
        q[i] = d + lorenzo_pred<NDIM>(q, i);
    }
    if (active) {
        const BlockOrigin bo = block_origin<NDIM>(g, b);
        using S = BlockShape<NDIM>;
        constexpr bool ROW32 = (S::BX * sizeof(T)) % 32 == 0;
        if (ROW32 && g.vec32 && interior_vec<T, NDIM>(g, bo)) {
            // 256-bit streaming stores (3D f64: one per row)
            constexpr int V32 = 32 / sizeof(T);
#pragma unroll
            for (int r = 0; r < S::BY * S::BZ; r++) {
                const int iy = r % S::BY, iz = r / S::BY;
                T *row = out + ((bo.z0 + iz) * g.ny + bo.y0 + iy) * g.nx + bo.x0;
#pragma unroll
                for (int u = 0; u < S::BX / V32; u++) {
                    T tmp[V32];
#pragma unroll
                    for (int k = 0; k < V32; k++) tmp[k] = dequantize(q[r * S::BX + u * V32 + k], K.s);
                    st32B_cs(row + u * V32, tmp);
                }
            }
        } else if (interior_vec<T, NDIM>(g, bo)) {
            using VT = typename Vec16<T>::type;
            constexpr int V = Vec16<T>::V;
#pragma unroll
            for (int r = 0; r < S::BY * S::BZ; r++) {
                const int iy = r % S::BY, iz = r / S::BY;
                VT *row = reinterpret_cast<VT *>(out + ((bo.z0 + iz) * g.ny + bo.y0 + iy) * g.nx + bo.x0);
#pragma unroll
                for (int v = 0; v < S::BX / V; v++) {
                    T tmp[V];
#pragma unroll
                    for (int k = 0; k < V; k++) tmp[k] = dequantize(q[r * S::BX + v * V + k], K.s);
                    // streaming (.cs) stores: 3D f32 512^3 4.13 -> 4.70 TB/s, f64 and
                    // 2D +-0 (profiles/ab_nd_cs_r01j.txt)
                    __stcs(row + v, *reinterpret_cast<VT *>(tmp));
                }
            }
        } else {
#pragma unroll
            for (int i = 0; i < LND; i++) {
                const uint64_t idx = nd_index<NDIM>(g, bo, i);
                if (idx != ~uint64_t(0)) out[idx] = dequantize(q[i], K.s);
            }
        }
    }
}

}  // namespace cszp2
