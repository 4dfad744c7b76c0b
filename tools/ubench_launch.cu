// Fixed cost of a kernel launch between two events, as the bench sees it (after a small-smem
// kernel): empty kernel, + 220 KB dynamic smem, + TMEM alloc/dealloc of 512 columns, grid 148.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ubench_launch tools/ubench_launch.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void busy(float* x, int n) {  // small-smem predecessor (stands in for the L2 flush)
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) x[i] = x[i] * 0.5f + 1.f;
}
template <bool TMEM>
__global__ void probe(int* out) {
    extern __shared__ unsigned char sm[];
    __shared__ unsigned tp;
    if (TMEM) {
        if (threadIdx.x < 32) {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((unsigned)__cvta_generic_to_shared(&tp)));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
        }
        __syncthreads();
        if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tp));
    }
    if (threadIdx.x == 0 && blockIdx.x == 0 && out) out[0] = (int)(size_t)sm;
}
int main() {
    float* x; int* o;
    cudaMalloc(&x, 64 << 20); cudaMalloc(&o, 16);
    cudaFuncSetAttribute(probe<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
    cudaFuncSetAttribute(probe<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    struct { const char* n; int smem; bool tm; int threads; } cs[] = {
        {"empty, 0 smem, 128 thr", 0, false, 128}, {"empty, 220 KB smem, 384 thr", 220 * 1024, false, 384},
        {"TMEM 512 alloc, 220 KB smem, 384 thr", 220 * 1024, true, 384}, {"TMEM 512, 220 KB, 640 thr", 220 * 1024, true, 640}};
    for (auto& c : cs) {
        float tot = 0; int K = 50;
        for (int it = 0; it < K + 5; ++it) {
            busy<<<(16 << 20) / 256, 256>>>(x, 16 << 20);
            cudaEventRecord(a);
            if (c.tm) probe<true><<<148, c.threads, c.smem>>>(o); else probe<false><<<148, c.threads, c.smem>>>(o);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms = -1; cudaError_t e_ = cudaEventElapsedTime(&ms, a, b); if (e_ != cudaSuccess && it == 5) printf("err %s\n", cudaGetErrorString(e_));
            if (it >= 5) tot += ms;
        }
        printf("%-40s %.2f us\n", c.n, tot / K * 1e3);
    }
    // two dependent kernels back to back (the chain), each with 220 KB smem + TMEM
    float tot = 0; int K = 50;
    for (int it = 0; it < K + 5; ++it) {
        busy<<<(16 << 20) / 256, 256>>>(x, 16 << 20);
        cudaEventRecord(a);
        probe<true><<<148, 384, 220 * 1024>>>(o);
        probe<true><<<148, 512, 220 * 1024>>>(o);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = -1; cudaError_t e_ = cudaEventElapsedTime(&ms, a, b); if (e_ != cudaSuccess && it == 5) printf("err %s\n", cudaGetErrorString(e_));
        if (it >= 5) tot += ms;
    }
    printf("%-40s %.2f us\n", "two TMEM kernels back to back", tot / K * 1e3);
    // the same pair with programmatic dependent launch on the second
    auto pdl = [&](int thr) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = 148; cfg.blockDim = thr; cfg.dynamicSmemBytes = 220 * 1024; cfg.stream = 0;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = at; cfg.numAttrs = 1;
        cudaLaunchKernelEx(&cfg, probe<true>, o);
    };
    tot = 0;
    for (int it = 0; it < K + 5; ++it) {
        busy<<<(16 << 20) / 256, 256>>>(x, 16 << 20);
        cudaEventRecord(a);
        probe<true><<<148, 384, 220 * 1024>>>(o);
        pdl(512);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = -1; cudaEventElapsedTime(&ms, a, b);
        if (it >= 5) tot += ms;
    }
    printf("%-40s %.2f us\n", "pair, second with PDL attribute", tot / K * 1e3);
    // CUDA graph of one kernel / of the pair
    cudaStream_t s; cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    for (int npair = 1; npair <= 2; ++npair) {
        cudaGraph_t g; cudaGraphExec_t ge;
        cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
        probe<true><<<148, 384, 220 * 1024, s>>>(o);
        if (npair == 2) probe<true><<<148, 512, 220 * 1024, s>>>(o);
        cudaStreamEndCapture(s, &g);
        cudaGraphInstantiate(&ge, g, 0);
        tot = 0;
        for (int it = 0; it < K + 5; ++it) {
            busy<<<(16 << 20) / 256, 256, 0, s>>>(x, 16 << 20);
            cudaEventRecord(a, s);
            cudaGraphLaunch(ge, s);
            cudaEventRecord(b, s);
            cudaEventSynchronize(b);
            float ms = -1; cudaEventElapsedTime(&ms, a, b);
            if (it >= 5) tot += ms;
        }
        printf("graph of %d TMEM kernel(s)                %.2f us\n", npair, tot / K * 1e3);
    }
    // event pair with nothing in between
    tot = 0;
    for (int it = 0; it < K + 5; ++it) {
        busy<<<(16 << 20) / 256, 256>>>(x, 16 << 20);
        cudaEventRecord(a);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = -1; cudaEventElapsedTime(&ms, a, b);
        if (it >= 5) tot += ms;
    }
    printf("%-40s %.2f us\n", "events only", tot / K * 1e3);
    return 0;
}
