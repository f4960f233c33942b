// Microbenchmark (dev aid): read throughput of persistent CTAs that stream 32 KiB
// tiles from HBM into shared memory, C CTAs per SM, K buffers per CTA, with a
// simulated per-tile compute time D (ns, spin on %globaltimer) after each tile.
// Load engines (M):
//   0  one 1D bulk TMA copy of 32 KiB (cp.async.bulk)
//   1  eight 1D bulk copies of 4 KiB, issued by 8 lanes
//   2  2D tensor TMA, 256 rows x 128 B box, 128-byte swizzle (the compressor's load)
//   3  cooperative cp.async.cg 16 B (LDGSTS) by all 256 threads, mbarrier completion
//   4  cooperative ld.global.cs 16 B into registers, then st.shared (no async copy)
// Answers: which engine and how many bytes in flight per SM the B200 HBM needs.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_inflight tma_inflight.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda.h>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t c) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void cpasync_arrive(uint64_t *b) {
    asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t par) {
    uint32_t ok;
    do {
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0,1,0,p;\n\t}"
                     : "=r"(ok) : "r"(smem_u32(b)), "r"(par) : "memory");
    } while (!ok);
}
__device__ __forceinline__ void bulk_load(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *map, int x, int y, uint64_t *bar) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"(smem_u32(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void cp_async16(void *dst, const void *src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ uint64_t gtimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

constexpr uint32_t TILE = 32768;

// issue the load of tile t into buffer k; every thread calls it (engines 3, 4 are cooperative)
__device__ __forceinline__ void issue(int M, const uint8_t *in, const CUtensorMap *map, uint8_t *dst,
                                      uint64_t *bar, unsigned t, unsigned ntiles) {
    const int tid = threadIdx.x;
    if (t >= ntiles) {
        if (M >= 3) { mbar_arrive(bar); } else if (tid == 0) mbar_expect_tx(bar, 0);
        return;
    }
    const uint8_t *src = in + (uint64_t)t * TILE;
    if (M == 0) {
        if (tid == 0) { mbar_expect_tx(bar, TILE); bulk_load(dst, src, TILE, bar); }
    } else if (M == 1) {
        if (tid == 0) mbar_expect_tx(bar, TILE);
        __syncwarp();
        if (tid < 8) bulk_load(dst + tid * 4096, src + tid * 4096, 4096, bar);
    } else if (M == 2) {
        if (tid == 0) { mbar_expect_tx(bar, TILE); tma_load_2d(dst, map, 0, (int)(t * 256), bar); }
    } else if (M == 3) {
#pragma unroll
        for (int c = 0; c < 8; c++) cp_async16(dst + (c * 256 + tid) * 16, src + (c * 256 + tid) * 16);
        cpasync_arrive(bar);
    } else {
        uint4 v[8];
#pragma unroll
        for (int c = 0; c < 8; c++) v[c] = __ldcs(reinterpret_cast<const uint4 *>(src) + c * 256 + tid);
#pragma unroll
        for (int c = 0; c < 8; c++) reinterpret_cast<uint4 *>(dst)[c * 256 + tid] = v[c];
        mbar_arrive(bar);
    }
}

__global__ void __launch_bounds__(256) stream_kernel(const __grid_constant__ CUtensorMap map, const uint8_t *in,
                                                     unsigned ntiles, int K, int D, int M, unsigned *ticket,
                                                     unsigned long long *sink) {
    extern __shared__ uint8_t raw[];
    uint8_t *buf = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(raw) + 1023) & ~uintptr_t(1023));
    __shared__ uint64_t full[8];
    __shared__ unsigned s_t[8];
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int k = 0; k < K; k++) mbar_init(&full[k], M >= 3 ? 256 : 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int k = 0; k < K; k++) s_t[k] = atomicAdd(ticket, 1u);
    }
    __syncthreads();
    for (int k = 0; k < K; k++) issue(M, in, &map, buf + k * TILE, &full[k], s_t[k], ntiles);
    uint32_t acc = 0;
    for (uint32_t it = 0;; it++) {
        const int k = it % K;
        mbar_wait(&full[k], (it / K) & 1);
        const unsigned t = s_t[k];
        if (t >= ntiles) break;
        const uint4 *p = reinterpret_cast<const uint4 *>(buf + k * TILE + tid * 128);
#pragma unroll
        for (int c = 0; c < 8; c++) { uint4 v = p[c ^ (tid & 7)]; acc += v.x ^ v.y ^ v.z ^ v.w; }
        __syncthreads();  // buffer free, everyone has read s_t[k]
        if (tid == 0) s_t[k] = atomicAdd(ticket, 1u);
        __syncthreads();
        issue(M, in, &map, buf + k * TILE, &full[k], s_t[k], ntiles);
        if (D > 0) {
            const uint64_t t0 = gtimer();
            while (gtimer() - t0 < (uint64_t)D) { acc = acc * 1664525u + 1013904223u; }
        }
    }
    if (acc == 0x12345678u) atomicAdd(sink, 1ull);
}

// write side: CTAs bulk-store a 32 KiB shared buffer to consecutive tiles, K groups in flight
__global__ void __launch_bounds__(256) store_kernel(uint8_t *out, unsigned ntiles, int K, int D, unsigned *ticket) {
    extern __shared__ uint8_t raw[];
    uint8_t *buf = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(raw) + 1023) & ~uintptr_t(1023));
    __shared__ unsigned s_t;
    for (int i = threadIdx.x; i < (int)(TILE / 4); i += blockDim.x) reinterpret_cast<uint32_t *>(buf)[i] = i;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    while (true) {
        if (threadIdx.x == 0) s_t = atomicAdd(ticket, 1u);
        __syncthreads();
        const unsigned t = s_t;
        __syncthreads();
        if (t >= ntiles) break;
        if (threadIdx.x == 0) {
            asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(out + (uint64_t)t * TILE),
                         "r"(smem_u32(buf)), "r"(TILE) : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            if (K <= 1) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            else if (K == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
            else asm volatile("cp.async.bulk.wait_group.read 3;" ::: "memory");
        }
        if (D > 0) {
            const uint64_t t0 = gtimer();
            while (gtimer() - t0 < (uint64_t)D) {}
        }
    }
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main(int argc, char **argv) {
    const uint64_t bytes = (argc > 1 ? strtoull(argv[1], 0, 0) : (8ull << 30));
    const unsigned ntiles = (unsigned)(bytes / TILE);
    uint8_t *in;
    unsigned *ticket;
    unsigned long long *sink;
    cudaMalloc(&in, (uint64_t)ntiles * TILE);
    cudaMemset(in, 1, (uint64_t)ntiles * TILE);
    cudaMalloc(&ticket, 4);
    cudaMalloc(&sink, 8);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaFuncSetAttribute(stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 7 * TILE);
    // 2D view: rows of 128 B (32 f32), 256 rows per tile
    void *fp = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &q);
    auto enc = reinterpret_cast<CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                             const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill)>(fp);
    CUtensorMap map;
    cuuint64_t dims[2] = {32, (cuuint64_t)ntiles * 256};
    cuuint64_t strides[1] = {128};
    cuuint32_t box[2] = {32, 256}, es[2] = {1, 1};
    CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, in, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r) printf("tensor map error %d\n", (int)r);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    printf("bytes %.2f GiB, %d SMs\n", (double)ntiles * TILE / 1073741824.0, sms);
    {
        cudaFuncSetAttribute(store_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, TILE + 1024);
        for (int C : {2, 3, 4, 6})
            for (int K : {1, 2, 4})
                for (int D : {0, 1500}) {
                    float best = 1e9;
                    for (int rep = 0; rep < 3; rep++) {
                        cudaMemset(ticket, 0, 4);
                        cudaEventRecord(e0);
                        store_kernel<<<sms * C, 256, TILE + 1024>>>(in, ntiles, K, D, ticket);
                        cudaEventRecord(e1);
                        cudaEventSynchronize(e1);
                        float ms;
                        cudaEventElapsedTime(&ms, e0, e1);
                        if (ms < best) best = ms;
                    }
                    printf("store     C=%d K=%d D=%4d ns: %7.1f GB/s %s\n", C, K, D, (double)ntiles * TILE / best / 1e6,
                           cudaGetErrorString(cudaGetLastError()));
                }
        float best = 1e9;
        for (int rep = 0; rep < 3; rep++) {
            cudaEventRecord(e0);
            cudaMemsetAsync(in, rep, (uint64_t)ntiles * TILE);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        printf("cudaMemset: %7.1f GB/s\n", (double)ntiles * TILE / best / 1e6);
        if (argc > 2) return 0;
    }
    const char *names[] = {"bulk32K", "bulk8x4K", "tensor2D", "cp.async16", "ldg16"};
    const int CK[][2] = {{3, 1}, {3, 2}, {2, 2}, {2, 3}, {4, 1}, {6, 1}};
    const int Ds[] = {0, 1500};
    for (int M = 0; M < 5; M++)
        for (auto &ck : CK)
            for (int D : Ds) {
                const int C = ck[0], K = ck[1];
                float best = 1e9;
                for (int rep = 0; rep < 3; rep++) {
                    cudaMemset(ticket, 0, 4);
                    cudaEventRecord(e0);
                    stream_kernel<<<sms * C, 256, K * TILE + 1024>>>(map, in, ntiles, K, D, M, ticket, sink);
                    cudaEventRecord(e1);
                    cudaEventSynchronize(e1);
                    float ms;
                    cudaEventElapsedTime(&ms, e0, e1);
                    if (ms < best) best = ms;
                }
                cudaError_t err = cudaGetLastError();
                printf("%-10s C=%d K=%d inflight/SM=%3d KiB D=%4d ns: %7.1f GB/s %s\n", names[M], C, K, C * K * 32, D,
                       (double)ntiles * TILE / best / 1e6, err ? cudaGetErrorString(err) : "");
            }
    return 0;
}
