// cszp2_api.cu — C ABI (include/cszp2.h) over the sm_100a kernels in kernels.cuh.
// Argument validation, stream geometry (FORMAT.md §2), tensor-map encoding and
// launches. No compute happens on the host.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <utility>

#include "cszp2.h"
#include "kernels.cuh"
#include "kernels_nd.cuh"

using namespace cszp2;

namespace {

inline cudaStream_t S(void *s) { return reinterpret_cast<cudaStream_t>(s); }

Geom geometry(uint64_t n) {
    Geom g;
    g.n = n;
    g.nb = (n + L - 1) / L;
    g.nfull = n / L;
    g.T = (g.nb + BPT - 1) / BPT;
    g.O = roundup16(64 + 8 * g.T);
    g.D = roundup16(g.O + g.nb);
    return g;
}

bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

int wsize(int dtype) { return dtype == CSZP2_F32 ? 4 : (dtype == CSZP2_F64 ? 8 : 0); }

PFN_cuTensorMapEncodeTiled_v12000 encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) ==
                cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    });
    return fn;
}

// Dense value side of a tile as a 2D tensor of 128-byte rows (one f32 block or
// half an f64 block per row), box = 256 rows, 128-byte swizzle.
int make_tmap(CUtensorMap *m, const void *base, int dtype, uint64_t nfull) {
    std::memset(m, 0, sizeof(*m));
    if (nfull == 0) return CSZP2_OK;  // kernels never touch the map
    auto enc = encoder();
    if (!enc) return CSZP2_ERR_CUDA;
    const bool f32 = dtype == CSZP2_F32;
    cuuint64_t dims[2] = {f32 ? 32ull : 16ull, f32 ? nfull : 2 * nfull};
    cuuint64_t strides[1] = {128};
    cuuint32_t box[2] = {f32 ? 32u : 16u, 256u};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(m, f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2,
                     const_cast<void *>(base), dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? CSZP2_OK : CSZP2_ERR_CUDA;
}

// Per-device launch state. cudaFuncSetAttribute and the occupancy query act on the
// current device's context, so both are cached per (kernel, device): a process that
// drives several GPUs gets the attribute set on each of them.
int current_device() {
    int d = 0;
    cudaGetDevice(&d);
    return d;
}
struct LaunchCache {
    int attr_rc = -1;  // -1: not yet set on this device
    int grid = 0;      // resident CTAs (occupancy x SMs) on this device
};
LaunchCache &launch_cache(const void *kernel, int dev) {
    static std::mutex mu;
    static std::map<std::pair<const void *, int>, LaunchCache> m;
    std::lock_guard<std::mutex> lk(mu);
    return m[{kernel, dev}];  // std::map references stay valid across inserts
}
// Opt the kernel into `bytes` of dynamic shared memory on the current device (once).
template <typename K>
int set_smem(K kernel, int bytes) {
    LaunchCache &c = launch_cache(reinterpret_cast<const void *>(kernel), current_device());
    if (c.attr_rc < 0)
        c.attr_rc = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes) == cudaSuccess
                        ? CSZP2_OK
                        : CSZP2_ERR_CUDA;
    return c.attr_rc;
}

int launch_status() { return cudaGetLastError() == cudaSuccess ? CSZP2_OK : CSZP2_ERR_CUDA; }

// stream bound without the 16-byte scratch tail (FORMAT.md §2)
uint64_t stream_bound(const Geom &g) { return roundup16(g.D + static_cast<uint64_t>(4 * L) * g.nb); }

int sm_count();
// zero bytes [from, to) of d_out (8-byte multiples) and the tile ticket at stream_bound
int zero_scratch(void *d_out, uint64_t from, uint64_t to, const Geom &g, cudaStream_t st) {
    const uint64_t words = (to - from) / 8;
    const uint64_t want = (words + 255) / 256;
    const uint64_t cap = 4ull * sm_count();
    const unsigned zg = static_cast<unsigned>(want < 1 ? 1 : (want > cap ? cap : want));
    uint8_t *o = static_cast<uint8_t *>(d_out);
    zero_scratch_kernel<<<zg, 256, 0, st>>>(reinterpret_cast<uint64_t *>(o + from), words,
                                            reinterpret_cast<uint4 *>(o + stream_bound(g)));
    return cudaGetLastError() == cudaSuccess ? CSZP2_OK : CSZP2_ERR_CUDA;
}

int sm_count() {
    int sms = 0;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, current_device()) != cudaSuccess || sms <= 0)
        sms = 148;
    return sms;
}

// persistent grid: every CTA resident (occupancy x SMs of the current device), never
// more than tiles
template <typename K>
unsigned persistent_grid(K kernel, int threads, int smem, uint64_t tiles) {
    LaunchCache &c = launch_cache(reinterpret_cast<const void *>(kernel), current_device());
    if (c.grid <= 0) {
        int per_sm = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, smem) != cudaSuccess ||
            per_sm < 1)
            per_sm = 1;
        c.grid = per_sm * sm_count();
    }
    const uint64_t t = tiles ? tiles : 1;
    return static_cast<unsigned>(t < static_cast<uint64_t>(c.grid) ? t : c.grid);
}

// Largest n of the 1D entry points: the dense side is a tensor of 128-byte rows (n/32
// rows for f32, n/16 for f64) and TMA coordinates are int32, so rows stay below 2^31.
constexpr uint64_t MAX_N = 1ull << 35;

int check_compress_args(const void *d_in, uint64_t n, int dtype, double eb, int eb_mode,
                        const void *d_out) {
    if (!wsize(dtype) || !d_out || (!d_in && n)) return CSZP2_ERR_ARG;
    if (eb_mode != CSZP2_EB_ABS && eb_mode != CSZP2_EB_REL) return CSZP2_ERR_ARG;
    if (!(eb > 0.0) || !std::isfinite(eb)) return CSZP2_ERR_ARG;
    if (!aligned16(d_out) || (n && !aligned16(d_in))) return CSZP2_ERR_ARG;
    if (n > MAX_N) return CSZP2_ERR_ARG;
    return CSZP2_OK;
}

template <typename T>
int launch_minmax(const void *d_in, uint64_t n, double lambda, void *d_out, cudaStream_t st,
                  double *range_out = nullptr) {
    const int sms = sm_count();
    const uint64_t nchunks = n * sizeof(T) / MM_CHUNK;
    if (nchunks >= static_cast<uint64_t>(sms)) {  // bulk-TMA streaming, 2 CTAs per SM
        constexpr int smem = MM_STAGES * MM_CHUNK;
        if (int rc = set_smem(minmax_kernel_tma<T>, smem)) return rc;
        const uint64_t want = 2ull * sms;
        const int grid = static_cast<int>(nchunks < want ? nchunks : want);
        minmax_kernel_tma<T><<<grid, 256, smem, st>>>(static_cast<const T *>(d_in), n, lambda,
                                                       static_cast<uint8_t *>(d_out), range_out);
        return launch_status();
    }
    const uint64_t nvec = n / (16 / sizeof(T));
    uint64_t want = (nvec + 255) / 256;
    int grid = static_cast<int>(want < 1 ? 1 : (want > (uint64_t)sms * 8 ? (uint64_t)sms * 8 : want));
    minmax_kernel<T><<<grid, 256, 0, st>>>(static_cast<const T *>(d_in), n, lambda,
                                            static_cast<uint8_t *>(d_out), range_out);
    return launch_status();
}

template <typename T, bool OUTLIER, int LOAD, int LBR = LB_PER_LANE>
int launch_compress_l(const void *d_in, const Geom &g, double eb, int eb_mode, int enc_mode,
                      void *d_out, uint64_t *d_out_bytes, cudaStream_t st, unsigned flags) {
    constexpr int smem = compress_smem_bytes<T>();
    if (int rc = set_smem(compress_kernel<T, OUTLIER, LOAD, LBR>, smem)) return rc;
    const unsigned grid = persistent_grid(compress_kernel<T, OUTLIER, LOAD, LBR>, NT_COMP, smem, g.T);
    unsigned *ticket = reinterpret_cast<unsigned *>(static_cast<uint8_t *>(d_out) + stream_bound(g));
    // the lookback descriptors (= the tile index, and its pad to O) and the tile ticket
    // start from zero on every encode, so encode can be repeated on one buffer
    // (FORMAT.md §2); skipped when the caller vouches that a prepare zeroed them
    if (!(flags & CSZP2_FLAG_PREPARED))
        if (int rc = zero_scratch(d_out, 64, g.O, g, st)) return rc;
    CUtensorMap map;
    int rc = make_tmap(&map, d_in, Traits<T>::DTYPE, g.nfull);
    if (rc) return rc;
    HdrStatic hs;
    hs.word1 = 1u | (static_cast<uint32_t>(Traits<T>::DTYPE) << 8) |
               (static_cast<uint32_t>(enc_mode) << 16) | (5u << 24);
    hs.eb_mode = static_cast<uint32_t>(eb_mode);
    hs.eb_user = eb;
    hs.flags = flags;
    compress_kernel<T, OUTLIER, LOAD, LBR><<<grid, NT_COMP, smem, st>>>(
        map, static_cast<const T *>(d_in), g, eb, eb_mode == CSZP2_EB_REL ? 1 : 0,
        static_cast<uint8_t *>(d_out), ticket, d_out_bytes, hs);
    return launch_status();
}

template <typename T, bool OUTLIER>
int launch_compress(const void *d_in, const Geom &g, double eb, int eb_mode, int enc_mode,
                    void *d_out, uint64_t *d_out_bytes, cudaStream_t st, unsigned flags) {
    if (flags & CSZP2_FLAG_LOAD_VEC)
        return launch_compress_l<T, OUTLIER, LOAD_VEC>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags);
    if (flags & CSZP2_FLAG_LOAD_SCALAR)
        return launch_compress_l<T, OUTLIER, LOAD_SCALAR>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags);
    // lookback window: 32 wide up to LB_NARROW_TILES tiles, 256 wide beyond (kernels.cuh)
    const bool narrow = (flags & CSZP2_FLAG_LB_NARROW) || (!(flags & CSZP2_FLAG_LB_WIDE) && g.T <= LB_NARROW_TILES);
    if (narrow)
        return launch_compress_l<T, OUTLIER, LOAD_TMA, 1>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags);
    return launch_compress_l<T, OUTLIER, LOAD_TMA>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags);
}

template <typename T>
int launch_decompress(const void *d_cmp, void *d_out, const Geom &g, int *d_status,
                      cudaStream_t st) {
    constexpr int smem = decompress_smem_bytes<T>();
    if (int rc = set_smem(decompress_kernel<T>, smem)) return rc;
    const unsigned grid = persistent_grid(decompress_kernel<T>, NT, smem, g.T);
    CUtensorMap map;
    int rc = make_tmap(&map, d_out, Traits<T>::DTYPE, g.nfull);
    if (rc) return rc;
    decompress_kernel<T><<<grid, NT, smem, st>>>(
        map, static_cast<const uint8_t *>(d_cmp), static_cast<T *>(d_out), g, d_status);
    return launch_status();
}

// ---- NEXT #3: multi-dimensional Lorenzo layouts (FORMAT.md §7)
// 0 on success; ARG for a bad ndim / extent
int geometry_nd(uint64_t nx, uint64_t ny, uint64_t nz, int ndim, GeomND *g) {
    if (ndim != 2 && ndim != 3) return CSZP2_ERR_ARG;
    if (ndim == 2) {
        if (nz != 1) return CSZP2_ERR_ARG;
    }
    if (nx >= (1ull << 32) || ny >= (1ull << 32) || nz >= (1ull << 32)) return CSZP2_ERR_ARG;
    const uint64_t b = ndim == 2 ? 8 : 4, bz = ndim == 2 ? 1 : 4;
    g->nx = nx;
    g->ny = ny;
    g->nz = nz;
    // n <= MAX_N = 2^35 for compression and decompression alike; checked without overflow
    if (nx && ny && nz && (nx * ny > MAX_N || nx * ny * nz / nz != nx * ny || nx * ny * nz > MAX_N))
        return CSZP2_ERR_ARG;
    g->n = nx * ny * nz;
    g->nbx = (nx + b - 1) / b;
    g->nby = (ny + b - 1) / b;
    g->nbz = (nz + bz - 1) / bz;
    g->nb = g->nbx * g->nby * g->nbz;
    g->T = (g->nb + BPT - 1) / BPT;
    g->O = roundup16(64 + 8 * g->T);
    g->D = roundup16(g->O + g->nb);
    g->dbx = make_fastdiv(static_cast<uint32_t>(g->nbx ? g->nbx : 1));
    g->dby = make_fastdiv(static_cast<uint32_t>(g->nby ? g->nby : 1));
    return CSZP2_OK;
}
uint64_t stream_bound_nd(const GeomND &g) { return roundup16(g.D + static_cast<uint64_t>(4 * LND) * g.nb); }

// byte offsets of the block rows (r = iy + by * iz) for the nD gathers / scatters
template <typename T, int NDIM>
void nd_rows(GeomND &g) {
    const uint64_t by = NDIM == 2 ? 8 : 4;
    for (int r = 0; r < 16; r++) g.roff[r] = ((r / by) * g.ny + (r % by)) * g.nx * sizeof(T);
    g.ystep = g.roff[1];
    g.zstep = NDIM == 3 ? g.roff[4] - g.roff[3] : 0;
    g.vec = (g.nx % (16 / sizeof(T))) == 0 ? 1u : 0u;
    g.vec32 = 0;  // set by the launch from the buffer it accesses
}

template <typename T, int NDIM, bool OUTLIER, int LBR>
int launch_compress_nd_w(const void *d_in, const GeomND &g0, double eb, int eb_mode, int enc_mode,
                         void *d_out, uint64_t *d_out_bytes, cudaStream_t st) {
    constexpr int smem = ND_RING + 64;
    GeomND g = g0;  // + the gather strides of this value type
    nd_rows<T, NDIM>(g);
    g.vec32 = (reinterpret_cast<uintptr_t>(d_in) % 32 == 0 && (g.nx * sizeof(T)) % 32 == 0) ? 1u : 0u;
    if (int rc = set_smem(compress_nd_kernel<T, NDIM, OUTLIER, LBR>, smem)) return rc;
    unsigned *ticket = reinterpret_cast<unsigned *>(static_cast<uint8_t *>(d_out) + stream_bound_nd(g));
    HdrStatic hs;
    hs.word1 = 1u | (static_cast<uint32_t>(Traits<T>::DTYPE) << 8) |
               (static_cast<uint32_t>(enc_mode) << 16) | (6u << 24);
    hs.eb_mode = static_cast<uint32_t>(eb_mode);
    hs.eb_user = eb;
    hs.flags = 0;
    const unsigned grid = persistent_grid(compress_nd_kernel<T, NDIM, OUTLIER, LBR>, NT_COMP, smem, g.T);
    compress_nd_kernel<T, NDIM, OUTLIER, LBR><<<grid, NT_COMP, smem, st>>>(
        static_cast<const T *>(d_in), g, eb, eb_mode == CSZP2_EB_REL ? 1 : 0,
        static_cast<uint8_t *>(d_out), ticket, d_out_bytes, hs);
    return launch_status();
}
template <typename T, int NDIM, bool OUTLIER>
int launch_compress_nd(const void *d_in, const GeomND &g, double eb, int eb_mode, int enc_mode,
                       void *d_out, uint64_t *d_out_bytes, cudaStream_t st, unsigned flags) {
    // lookback window: 32 wide up to LB_NARROW_TILES tiles, 256 wide beyond (kernels.cuh),
    // unless forced by CSZP2_FLAG_LB_NARROW / CSZP2_FLAG_LB_WIDE
    if ((flags & CSZP2_FLAG_LB_NARROW) || (!(flags & CSZP2_FLAG_LB_WIDE) && g.T <= LB_NARROW_TILES))
        return launch_compress_nd_w<T, NDIM, OUTLIER, 1>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st);
    return launch_compress_nd_w<T, NDIM, OUTLIER, LB_PER_LANE>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st);
}

template <typename T, int NDIM>
int launch_decompress_nd(const void *d_cmp, void *d_out, const GeomND &g0, int *d_status,
                         cudaStream_t st) {
    if constexpr (sizeof(T) == 8) {  // f64: one CTA per tile (kernels_nd.cuh, decompress_nd_tile_kernel)
        constexpr int smem = ND_STAGE + 64;
        if (int rc = set_smem(decompress_nd_tile_kernel<T, NDIM>, smem)) return rc;
        GeomND g = g0;
        g.vec32 = (reinterpret_cast<uintptr_t>(d_out) % 32 == 0 && (g.nx * sizeof(T)) % 32 == 0) ? 1u : 0u;
        const unsigned grid = static_cast<unsigned>(g.T ? g.T : 1);
        decompress_nd_tile_kernel<T, NDIM><<<grid, NT, smem, st>>>(static_cast<const uint8_t *>(d_cmp),
                                                                   static_cast<T *>(d_out), g, d_status);
        return launch_status();
    } else {
        constexpr int smem = ND_DRING + 64;
        if (int rc = set_smem(decompress_nd_kernel<T, NDIM>, smem)) return rc;
        GeomND g = g0;
        nd_rows<T, NDIM>(g);
        g.vec32 = (reinterpret_cast<uintptr_t>(d_out) % 32 == 0 && (g.nx * sizeof(T)) % 32 == 0) ? 1u : 0u;
        const unsigned grid = persistent_grid(decompress_nd_kernel<T, NDIM>, NT, smem, g.T);
        decompress_nd_kernel<T, NDIM><<<grid, NT, smem, st>>>(static_cast<const uint8_t *>(d_cmp),
                                                              static_cast<T *>(d_out), g, d_status);
        return launch_status();
    }
}

template <typename T>
int dispatch_compress_nd(const void *d_in, const GeomND &g, int ndim, double eb, int eb_mode,
                         int enc_mode, void *d_out, uint64_t *d_out_bytes, cudaStream_t st, unsigned flags) {
    const bool o = enc_mode == CSZP2_ENC_OUTLIER;
    if (ndim == 2)
        return o ? launch_compress_nd<T, 2, true>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags)
                 : launch_compress_nd<T, 2, false>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags);
    return o ? launch_compress_nd<T, 3, true>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags)
             : launch_compress_nd<T, 3, false>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags);
}

}  // namespace

extern "C" {

const char *cszp2_version(void) { return "cszp2 1.0 sm_100a"; }

#ifdef CSZP2_TRACE
int cszp2_debug_set_trace(void *d_buf) {
    return cudaMemcpyToSymbol(g_trace, &d_buf, sizeof(void *)) == cudaSuccess ? 0 : 2;
}
#endif

uint64_t cszp2_compress_bound(uint64_t n, int dtype) {
    if (!wsize(dtype)) return 0;
    // the stream's worst case plus 16 bytes of scratch (the compression ticket)
    return stream_bound(geometry(n)) + 16;
}

int cszp2_compress_prepare(const void *d_in, uint64_t n, int dtype, double eb, int eb_mode,
                           void *d_out, void *stream) {
    int rc = check_compress_args(d_in, n, dtype, eb, eb_mode, d_out);
    if (rc) return rc;
    // the header (REL's reduction scratch and eb_abs), the tile index and the ticket:
    // one launch, so that cszp2_compress's encode needs none (CSZP2_FLAG_PREPARED)
    if (int zr = zero_scratch(d_out, 0, geometry(n).O, geometry(n), S(stream))) return zr;
    if (eb_mode == CSZP2_EB_REL)
        return dtype == CSZP2_F32 ? launch_minmax<float>(d_in, n, eb, d_out, S(stream))
                                  : launch_minmax<double>(d_in, n, eb, d_out, S(stream));
    return CSZP2_OK;
}

int cszp2_value_range(const void *d_in, uint64_t n, int dtype, double *d_work, void *stream) {
    if (!wsize(dtype) || !d_work || (!d_in && n)) return CSZP2_ERR_ARG;
    if ((n && !aligned16(d_in)) || !aligned16(d_work) || n > MAX_N) return CSZP2_ERR_ARG;
    // d_work[0..1]: the result; bytes 32..63: the reduction's header-shaped scratch
    if (cudaMemsetAsync(d_work, 0, 8 * sizeof(double), S(stream)) != cudaSuccess) return CSZP2_ERR_CUDA;
    return dtype == CSZP2_F32 ? launch_minmax<float>(d_in, n, 1.0, d_work, S(stream), d_work)
                              : launch_minmax<double>(d_in, n, 1.0, d_work, S(stream), d_work);
}

int cszp2_compress_prepare_range(const void *d_in, uint64_t n, int dtype, double eb,
                                 const double *d_range, void *d_out, void *stream) {
    int rc = check_compress_args(d_in, n, dtype, eb, CSZP2_EB_REL, d_out);
    if (rc) return rc;
    if (!d_range || !aligned16(d_range)) return CSZP2_ERR_ARG;
    if (int zr = zero_scratch(d_out, 0, geometry(n).O, geometry(n), S(stream))) return zr;
    eb_from_range_kernel<<<1, 1, 0, S(stream)>>>(d_range, eb, static_cast<uint8_t *>(d_out));
    return launch_status();
}

int cszp2_compress_encode_ex(const void *d_in, uint64_t n, int dtype, double eb, int eb_mode,
                             int enc_mode, void *d_out, uint64_t *d_out_bytes, unsigned flags,
                             void *stream) {
    int rc = check_compress_args(d_in, n, dtype, eb, eb_mode, d_out);
    if (rc) return rc;
    if (enc_mode != CSZP2_ENC_PLAIN && enc_mode != CSZP2_ENC_OUTLIER) return CSZP2_ERR_ARG;
    if (flags & ~(CSZP2_FLAG_CHAINED_SCAN | CSZP2_FLAG_LOAD_VEC | CSZP2_FLAG_LOAD_SCALAR | CSZP2_FLAG_PREPARED |
                  CSZP2_FLAG_LB_WIDE | CSZP2_FLAG_LB_NARROW))
        return CSZP2_ERR_ARG;
    if ((flags & CSZP2_FLAG_LOAD_VEC) && (flags & CSZP2_FLAG_LOAD_SCALAR)) return CSZP2_ERR_ARG;
    if ((flags & CSZP2_FLAG_LB_WIDE) && (flags & CSZP2_FLAG_LB_NARROW)) return CSZP2_ERR_ARG;
    Geom g = geometry(n);
    cudaStream_t st = S(stream);
    if (dtype == CSZP2_F32)
        return enc_mode == CSZP2_ENC_OUTLIER
                   ? launch_compress<float, true>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags)
                   : launch_compress<float, false>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags);
    return enc_mode == CSZP2_ENC_OUTLIER
               ? launch_compress<double, true>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags)
               : launch_compress<double, false>(d_in, g, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags);
}

int cszp2_compress_encode(const void *d_in, uint64_t n, int dtype, double eb, int eb_mode,
                          int enc_mode, void *d_out, uint64_t *d_out_bytes, void *stream) {
    return cszp2_compress_encode_ex(d_in, n, dtype, eb, eb_mode, enc_mode, d_out, d_out_bytes, 0u,
                                    stream);
}

int cszp2_compress(const void *d_in, uint64_t n, int dtype, double eb, int eb_mode, int enc_mode,
                   void *d_out, uint64_t *d_out_bytes, void *stream) {
    if (enc_mode != CSZP2_ENC_PLAIN && enc_mode != CSZP2_ENC_OUTLIER) return CSZP2_ERR_ARG;
    int rc = cszp2_compress_prepare(d_in, n, dtype, eb, eb_mode, d_out, stream);
    if (rc) return rc;
    return cszp2_compress_encode_ex(d_in, n, dtype, eb, eb_mode, enc_mode, d_out, d_out_bytes, CSZP2_FLAG_PREPARED,
                                    stream);
}

int cszp2_decompress(const void *d_cmp, void *d_out, uint64_t n, int dtype, int *d_status,
                     void *stream) {
    if (!wsize(dtype) || !d_cmp || (!d_out && n)) return CSZP2_ERR_ARG;
    if (!aligned16(d_cmp) || (n && !aligned16(d_out))) return CSZP2_ERR_ARG;
    if (n > MAX_N) return CSZP2_ERR_ARG;
    Geom g = geometry(n);
    return dtype == CSZP2_F32 ? launch_decompress<float>(d_cmp, d_out, g, d_status, S(stream))
                              : launch_decompress<double>(d_cmp, d_out, g, d_status, S(stream));
}

uint64_t cszp2_decompress_scratch_bytes(uint64_t n) {
    const Geom g = geometry(n);
    return 8 * (g.T ? g.T : 1) + 16;  // descriptors + ticket
}

int cszp2_decompress_tilewise(const void *d_cmp, void *d_out, uint64_t n, int dtype, int locate,
                              void *d_scratch, int *d_status, void *stream) {
    if (!wsize(dtype) || !d_cmp || !d_scratch || (!d_out && n)) return CSZP2_ERR_ARG;
    if (locate != CSZP2_LOCATE_INDEX && locate != CSZP2_LOCATE_LOOKBACK) return CSZP2_ERR_ARG;
    if (!aligned16(d_cmp) || (n && !aligned16(d_out)) || n > MAX_N) return CSZP2_ERR_ARG;
    const Geom g = geometry(n);
    cudaStream_t st = S(stream);
    if (cudaMemsetAsync(d_scratch, 0, cszp2_decompress_scratch_bytes(n), st) != cudaSuccess)
        return CSZP2_ERR_CUDA;
    const unsigned grid = static_cast<unsigned>(g.T ? g.T : 1);
    uint64_t *scr = static_cast<uint64_t *>(d_scratch);
    const uint8_t *c = static_cast<const uint8_t *>(d_cmp);
    const bool lb = locate == CSZP2_LOCATE_LOOKBACK;
    if (dtype == CSZP2_F32) {
        float *o = static_cast<float *>(d_out);
        if (lb)
            decompress_tilewise_kernel<float, true><<<grid, NT, 0, st>>>(c, o, g, scr, d_status);
        else
            decompress_tilewise_kernel<float, false><<<grid, NT, 0, st>>>(c, o, g, scr, d_status);
    } else {
        double *o = static_cast<double *>(d_out);
        if (lb)
            decompress_tilewise_kernel<double, true><<<grid, NT, 0, st>>>(c, o, g, scr, d_status);
        else
            decompress_tilewise_kernel<double, false><<<grid, NT, 0, st>>>(c, o, g, scr, d_status);
    }
    return launch_status();
}

int cszp2_decompress_range(const void *d_cmp, uint64_t n, int dtype, uint64_t first,
                           uint64_t count, void *d_out, int *d_status, void *stream) {
    if (!wsize(dtype) || !d_cmp || (!d_out && count)) return CSZP2_ERR_ARG;
    if (!aligned16(d_cmp) || n > MAX_N || first > n || count > n - first) return CSZP2_ERR_ARG;
    if (count == 0) return CSZP2_OK;
    Geom g = geometry(n);
    const uint64_t t0 = (first / L) / BPT, t1 = ((first + count - 1) / L) / BPT;
    const unsigned grid = static_cast<unsigned>(t1 - t0 + 1);
    if (dtype == CSZP2_F32)
        decompress_range_kernel<float><<<grid, NT, 0, S(stream)>>>(
            static_cast<const uint8_t *>(d_cmp), static_cast<float *>(d_out), g, first, count, t0, d_status);
    else
        decompress_range_kernel<double><<<grid, NT, 0, S(stream)>>>(
            static_cast<const uint8_t *>(d_cmp), static_cast<double *>(d_out), g, first, count, t0, d_status);
    return launch_status();
}

int cszp2_read_header(const void *d_cmp, cszp2_header *h, void *stream) {
    if (!d_cmp || !h) return CSZP2_ERR_ARG;
    uint8_t raw[64];
    if (cudaMemcpyAsync(raw, d_cmp, 64, cudaMemcpyDeviceToHost, S(stream)) != cudaSuccess ||
        cudaStreamSynchronize(S(stream)) != cudaSuccess)
        return CSZP2_ERR_CUDA;
    std::memcpy(&h->magic, raw + 0, 4);
    h->version = raw[4];
    h->dtype = raw[5];
    h->enc_mode = raw[6];
    h->log2L = raw[7];
    h->eb_mode = raw[8];
    h->status = raw[9];
    std::memcpy(&h->blocks_per_tile, raw + 10, 2);
    std::memcpy(&h->n, raw + 16, 8);
    std::memcpy(&h->eb, raw + 24, 8);
    std::memcpy(&h->eb_abs, raw + 32, 8);
    std::memcpy(&h->payload_bytes, raw + 40, 8);
    std::memcpy(&h->total_bytes, raw + 48, 8);
    return CSZP2_OK;
}

int cszp2_compress_host(const void *h_in, uint64_t n, int dtype, double eb, int eb_mode,
                        int enc_mode, void *d_in_work, void *d_out_work, void *h_out,
                        uint64_t h_out_cap, uint64_t *h_out_bytes, void *stream) {
    if (!h_out || !h_out_bytes || (!h_in && n)) return CSZP2_ERR_ARG;
    const int w = wsize(dtype);
    if (!w) return CSZP2_ERR_ARG;
    if (n && cudaMemcpyAsync(d_in_work, h_in, n * w, cudaMemcpyHostToDevice, S(stream)) != cudaSuccess)
        return CSZP2_ERR_CUDA;
    int rc = cszp2_compress(d_in_work, n, dtype, eb, eb_mode, enc_mode, d_out_work, nullptr, stream);
    if (rc) return rc;
    uint64_t total = 0;  // the stream's own header holds its size (FORMAT.md §3)
    if (cudaMemcpyAsync(&total, static_cast<uint8_t *>(d_out_work) + 48, 8, cudaMemcpyDeviceToHost,
                        S(stream)) != cudaSuccess ||
        cudaStreamSynchronize(S(stream)) != cudaSuccess)
        return CSZP2_ERR_CUDA;
    if (total > h_out_cap) return CSZP2_ERR_ARG;
    if (cudaMemcpyAsync(h_out, d_out_work, total, cudaMemcpyDeviceToHost, S(stream)) != cudaSuccess ||
        cudaStreamSynchronize(S(stream)) != cudaSuccess)
        return CSZP2_ERR_CUDA;
    *h_out_bytes = total;
    return CSZP2_OK;
}

int cszp2_decompress_host(const void *h_cmp, uint64_t cmp_bytes, void *d_cmp_work,
                          void *d_out_work, void *h_out, uint64_t n, int dtype, int *d_status,
                          void *stream) {
    const int w = wsize(dtype);
    if (!w || !h_cmp || !d_cmp_work || (n && (!h_out || !d_out_work))) return CSZP2_ERR_ARG;
    if (cudaMemcpyAsync(d_cmp_work, h_cmp, cmp_bytes, cudaMemcpyHostToDevice, S(stream)) != cudaSuccess)
        return CSZP2_ERR_CUDA;
    int rc = cszp2_decompress(d_cmp_work, d_out_work, n, dtype, d_status, stream);
    if (rc) return rc;
    if (n && cudaMemcpyAsync(h_out, d_out_work, n * w, cudaMemcpyDeviceToHost, S(stream)) != cudaSuccess)
        return CSZP2_ERR_CUDA;
    int st = 0;
    if (d_status && cudaMemcpyAsync(&st, d_status, 4, cudaMemcpyDeviceToHost, S(stream)) != cudaSuccess)
        return CSZP2_ERR_CUDA;
    if (cudaStreamSynchronize(S(stream)) != cudaSuccess) return CSZP2_ERR_CUDA;
    return st;
}

uint64_t cszp2_compress_bound_nd(uint64_t nx, uint64_t ny, uint64_t nz, int ndim, int dtype) {
    GeomND g;
    if (!wsize(dtype) || geometry_nd(nx, ny, nz, ndim, &g)) return 0;
    return stream_bound_nd(g) + 16;  // + the ticket scratch, as cszp2_compress_bound
}

int cszp2_compress_nd(const void *d_in, uint64_t nx, uint64_t ny, uint64_t nz, int ndim, int dtype,
                      double eb, int eb_mode, int enc_mode, void *d_out, uint64_t *d_out_bytes,
                      void *stream) {
    return cszp2_compress_nd_ex(d_in, nx, ny, nz, ndim, dtype, eb, eb_mode, enc_mode, d_out, d_out_bytes, 0u,
                                stream);
}

int cszp2_compress_nd_ex(const void *d_in, uint64_t nx, uint64_t ny, uint64_t nz, int ndim, int dtype,
                         double eb, int eb_mode, int enc_mode, void *d_out, uint64_t *d_out_bytes,
                         unsigned flags, void *stream) {
    GeomND g;
    if (flags & ~(CSZP2_FLAG_LB_WIDE | CSZP2_FLAG_LB_NARROW)) return CSZP2_ERR_ARG;
    if ((flags & CSZP2_FLAG_LB_WIDE) && (flags & CSZP2_FLAG_LB_NARROW)) return CSZP2_ERR_ARG;
    if (geometry_nd(nx, ny, nz, ndim, &g)) return CSZP2_ERR_ARG;
    if (enc_mode != CSZP2_ENC_PLAIN && enc_mode != CSZP2_ENC_OUTLIER) return CSZP2_ERR_ARG;
    int rc = check_compress_args(d_in, g.n, dtype, eb, eb_mode, d_out);
    if (rc) return rc;
    cudaStream_t st = S(stream);
    if (cudaMemsetAsync(d_out, 0, g.O, st) != cudaSuccess ||
        cudaMemsetAsync(static_cast<uint8_t *>(d_out) + stream_bound_nd(g), 0, 16, st) != cudaSuccess)
        return CSZP2_ERR_CUDA;
    if (eb_mode == CSZP2_EB_REL) {
        rc = dtype == CSZP2_F32 ? launch_minmax<float>(d_in, g.n, eb, d_out, st)
                                : launch_minmax<double>(d_in, g.n, eb, d_out, st);
        if (rc) return rc;
    }
    return dtype == CSZP2_F32
               ? dispatch_compress_nd<float>(d_in, g, ndim, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags)
               : dispatch_compress_nd<double>(d_in, g, ndim, eb, eb_mode, enc_mode, d_out, d_out_bytes, st, flags);
}

int cszp2_decompress_nd(const void *d_cmp, void *d_out, uint64_t nx, uint64_t ny, uint64_t nz, int ndim,
                        int dtype, int *d_status, void *stream) {
    GeomND g;
    if (!wsize(dtype) || !d_cmp || geometry_nd(nx, ny, nz, ndim, &g)) return CSZP2_ERR_ARG;
    if ((!d_out && g.n) || !aligned16(d_cmp) || (g.n && !aligned16(d_out))) return CSZP2_ERR_ARG;
    cudaStream_t st = S(stream);
    if (dtype == CSZP2_F32)
        return ndim == 2 ? launch_decompress_nd<float, 2>(d_cmp, d_out, g, d_status, st)
                         : launch_decompress_nd<float, 3>(d_cmp, d_out, g, d_status, st);
    return ndim == 2 ? launch_decompress_nd<double, 2>(d_cmp, d_out, g, d_status, st)
                     : launch_decompress_nd<double, 3>(d_cmp, d_out, g, d_status, st);
}

int cszp2_container_index(const uint64_t *d_sizes, int nparts, uint64_t *d_offsets,
                          void *stream) {
    if (!d_sizes || !d_offsets || nparts < 1) return CSZP2_ERR_ARG;
    container_index_kernel<<<1, 32, 0, S(stream)>>>(d_sizes, nparts, d_offsets);
    return launch_status();
}

}  // extern "C"

#ifdef CSZP2_WD
// debug build only: point the kernels' watchdog records at host-mapped memory
extern "C" int cszp2_debug_watch(void *p) {
    return cudaMemcpyToSymbol(cszp2::g_wd, &p, sizeof(p)) == cudaSuccess ? CSZP2_OK : CSZP2_ERR_CUDA;
}
#endif
