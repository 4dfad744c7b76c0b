// Does compute-sanitizer racecheck model mbarrier parity waits?  A textbook, correct handoff:
// warp 0 writes a shared buffer, __syncwarp, lane 0 arrives (release.cta) on `full`; warp 1 waits
// on `full` (try_wait.parity, acquire.cta) and reads it, then arrives on `empty`; warp 0 waits on
// `empty` before the next write.  Same pattern as the GEMM1 epilogue -> IR statistics ring
// (g1_body.cuh).  If racecheck reports RAW/WAR hazards here, they are tool false positives.
// nvcc -gencode arch=compute_100a,code=sm_100a -o ubench_racecheck_mbar tools/ubench_racecheck_mbar.cu
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void arrive(uint64_t* b)
{
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(sa(b)) : "memory");
}
__device__ __forceinline__ void wait(uint64_t* b, uint32_t ph)
{
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{\n\t.reg .pred P1;\n\tmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P1, [%1], %2;\n\t"
                     "selp.b32 %0, 1, 0, P1;\n\t}" : "=r"(ok) : "r"(sa(b)), "r"(ph) : "memory");
}

__global__ void handoff(float* out, int rounds)
{
    __shared__ float buf[128];
    __shared__ uint64_t full, empty;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&full)));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&empty)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    float acc = 0.f;
    for (int i = 0; i < rounds; ++i) {
        if (warp == 0) {
            if (i > 0) wait(&empty, (i - 1) & 1);
            for (int j = lane; j < 128; j += 32) buf[j] = i + j;
            __syncwarp();
            if (lane == 0) arrive(&full);
        } else {
            wait(&full, i & 1);
            for (int j = lane; j < 128; j += 32) acc += buf[j];
            __syncwarp();
            if (lane == 0) arrive(&empty);
        }
    }
    if (warp == 1) out[lane] = acc;
}

int main()
{
    float* d;
    cudaMalloc(&d, 128);
    handoff<<<1, 64>>>(d, 8);
    float h[32];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double want = 0;
    for (int i = 0; i < 8; ++i)
        for (int j = 0; j < 128; j += 32) want += i + j;  // lane 0's sum
    printf("mbarrier handoff: lane0 %.0f (expect %.0f) %s\n", h[0], want, h[0] == want ? "ok" : "WRONG");
    cudaFree(d);
    return 0;
}
