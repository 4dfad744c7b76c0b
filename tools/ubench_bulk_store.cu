// Microbenchmark: achievable HBM write bandwidth of cp.async.bulk shared->global stores on B200,
// as a function of store size, bulk-groups in flight per issuing warp, and issuing warps per CTA.
// (Ceiling of GEMM1's X' write path.)  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ub ubench_bulk_store.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int DEPTH>
__global__ void __launch_bounds__(512, 1) store_kernel(uint8_t* dst, size_t total, int chunk, int warps)
{
    extern __shared__ __align__(1024) uint8_t sm[];
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    for (int i = threadIdx.x; i < 65536; i += blockDim.x) sm[i] = (uint8_t)i;
    __syncthreads();
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (warp >= warps || lane != 0) return;
    const size_t n_chunks = total / chunk;
    uint8_t* src = sm + warp * (65536 / warps);
    for (size_t c = (size_t)blockIdx.x * warps + warp; c < n_chunks; c += (size_t)gridDim.x * warps) {
        asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(DEPTH - 1) : "memory");
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + c * chunk),
                     "r"(smem_u32(src)), "r"(chunk)
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

__global__ void stg_kernel(uint4* dst, size_t n)  // reference: plain coalesced vector stores
{
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        dst[i] = make_uint4((uint32_t)i, 1, 2, 3);
}

int main()
{
    const size_t total = 285ull << 20;
    uint8_t* d;
    cudaMalloc(&d, total);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    auto time = [&](auto launch) {
        launch();
        cudaDeviceSynchronize();
        float best = 1e9;
        for (int r = 0; r < 5; ++r) {
            cudaEventRecord(a);
            launch();
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            best = ms < best ? ms : best;
        }
        return total / (best * 1e-3) / 1e9;
    };
    printf("plain st.global.v4: %.0f GB/s\n", time([&] { stg_kernel<<<sms * 8, 256>>>((uint4*)d, total / 16); }));
    for (auto f : {store_kernel<1>, store_kernel<2>, store_kernel<4>})
        cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
    const int chunks[] = {4096, 8192, 16384, 32768};
    const int warpss[] = {1, 2, 4, 8, 16};
    for (int depth : {1, 2, 4})
        for (int chunk : chunks)
            for (int w : warpss) {
                if ((size_t)chunk * 1 > 65536 / w) continue;
                double gbs = time([&] {
                    if (depth == 1) store_kernel<1><<<sms, 512, 65536>>>(d, total, chunk, w);
                    if (depth == 2) store_kernel<2><<<sms, 512, 65536>>>(d, total, chunk, w);
                    if (depth == 4) store_kernel<4><<<sms, 512, 65536>>>(d, total, chunk, w);
                });
                printf("bulk store depth %d chunk %6d warps %2d: %6.0f GB/s (%d KB in flight/SM)\n", depth, chunk, w, gbs,
                       depth * chunk * w / 1024);
            }
    return 0;
}
