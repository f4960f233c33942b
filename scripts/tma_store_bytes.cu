// Microbenchmark + correctness probe (dev aid): TMA tensor stores of 256-byte uint8
// boxes from shared memory to ARBITRARY byte offsets in global memory (1D tensor map),
// as a possible replacement for the compression resolver's SIMT payload copy.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tsb scripts/tma_store_bytes.cu -lcuda
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

template <int SOFF>
__global__ void __launch_bounds__(128) k(const __grid_constant__ CUtensorMap map, uint64_t per, uint32_t off, int nbox, int reps) {
    __shared__ __align__(1024) uint8_t buf[16384 + 256];
    uint8_t *src = buf + SOFF;
    for (int i = threadIdx.x; i < nbox * 256; i += blockDim.x) src[i] = static_cast<uint8_t>((blockIdx.x * 131 + i * 7 + 1) & 0xFF);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int r = 0; r < reps; r++) {
            const uint64_t o = blockIdx.x * per + off;
            for (int b = 0; b < nbox; b++) {
                asm volatile("cp.async.bulk.tensor.1d.global.shared::cta.bulk_group [%0, {%1}], [%2];" ::"l"(&map),
                             "r"(static_cast<int>(o + 256ull * b)), "r"(smem_u32(src + 256 * b))
                             : "memory");
            }
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        }
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
}

int main() {
    setvbuf(stdout, nullptr, _IONBF, 0);
    const int grid = 444, nbox = 56;  // 14 KiB per CTA, like a cfg4a Plain tile
    const uint64_t per = nbox * 256 + 4096;
    const uint64_t N = grid * per + 4096;
    uint8_t *d;
    cudaMalloc(&d, N);
    PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaError_t ge = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", reinterpret_cast<void **>(&enc), cudaEnableDefault, &q);
    printf("entry point: %s q=%d fn=%p\n", cudaGetErrorString(ge), (int)q, (void *)enc);
    if (!enc) return 1;
    CUtensorMap map;
    cuuint64_t dims[1] = {N};
    cuuint32_t box[1] = {256}, es[1] = {1};
    cuuint64_t strides[1] = {1};
    CUresult cr = enc(&map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 1, d, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode rc=%d\n", (int)cr);
    for (uint32_t off : {0u, 1u, 7u, 13u, 128u + 5u}) {
        cudaMemset(d, 0xEE, N);
        k<0><<<grid, 128>>>(map, per, off, nbox, 1);
        cudaError_t e = cudaDeviceSynchronize();
        std::vector<uint8_t> h(N);
        cudaMemcpy(h.data(), d, N, cudaMemcpyDeviceToHost);
        long bad = 0;
        for (int c = 0; c < grid; c++) {
            for (uint64_t i = 0; i < per; i++) {
                uint64_t o = c * per + i;
                uint8_t want = 0xEE;
                if (i >= off && i < off + nbox * 256) want = static_cast<uint8_t>((c * 131 + (i - off) * 7 + 1) & 0xFF);
                if (h[o] != want) bad++;
            }
        }
        printf("off=%u err=%s mismatches=%ld\n", off, cudaGetErrorString(e), bad);
    }
    // source offsets that are 16- but not 128-byte aligned
    k<16><<<grid, 128>>>(map, per, 3, nbox, 1);
    printf("smem+16: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    cudaGetLastError();
    k<64><<<grid, 128>>>(map, per, 3, nbox, 1);
    printf("smem+64: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    cudaGetLastError();
    // throughput: reps rounds of 14 KiB per CTA
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (uint32_t off : {0u, 5u}) {
        k<0><<<grid, 128>>>(map, per, off, nbox, 4);
        cudaEventRecord(a);
        k<0><<<grid, 128>>>(map, per, off, nbox, 200);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("off=%u: %.1f GB/s of TMA byte-box stores (%.2f us per 14 KiB round per CTA)\n", off,
               grid * 200.0 * nbox * 256 / (ms * 1e6), ms * 1e3 / 200);
    }
    return 0;
}
