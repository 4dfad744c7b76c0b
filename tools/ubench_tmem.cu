// Microbenchmark: tcgen05.ld (TMEM -> registers) throughput per SM on one B200, for the 32x32b
// shape used by the GEMM1 epilogue, with 4 / 8 / 16 warps per CTA, alone and interleaved with the
// epilogue's MUFU.EX2 work -- is GEMM1's LS epilogue bound by TMEM reads, MUFU, or their sum?
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ubench_tmem_bin tools/ubench_tmem.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }

__device__ __forceinline__ void ffma2(float& a, float& b, float s, float c)
{
    unsigned long long x = ((unsigned long long)__float_as_uint(b) << 32) | __float_as_uint(a);
    unsigned long long sc = ((unsigned long long)__float_as_uint(s) << 32) | __float_as_uint(s);
    unsigned long long cc = ((unsigned long long)__float_as_uint(c) << 32) | __float_as_uint(c);
    asm("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(x) : "l"(sc), "l"(cc));
    a = __uint_as_float((unsigned)x); b = __uint_as_float((unsigned)(x >> 32));
}
__device__ __forceinline__ void fadd2(float& a, float& b, float x, float y)
{
    unsigned long long u = ((unsigned long long)__float_as_uint(b) << 32) | __float_as_uint(a);
    unsigned long long v = ((unsigned long long)__float_as_uint(y) << 32) | __float_as_uint(x);
    asm("add.rn.f32x2 %0, %0, %1;" : "+l"(u) : "l"(v));
    a = __uint_as_float((unsigned)u); b = __uint_as_float((unsigned)(u >> 32));
}
__device__ __forceinline__ uint32_t pk(float a, float b) { uint32_t r; asm("cvt.rn.f16x2.f32 %0, %2, %1;" : "=r"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ void ld32(uint32_t taddr, uint32_t (&r)[32])
{
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
        "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}

// MODE 0: tcgen05.ld only (4 x32 loads = 128 columns per iteration, one wait)
// MODE 1: tcgen05.ld + 128 ex2 per lane per iteration (the LS epilogue's mix)
// MODE 2: 128 ex2 per lane per iteration only
// MODE 3: ld + the full LS math of the GEMM1 epilogue (max, FFMA2, ex2, FADD2, fp16 pack, st.shared)
template <int MODE>
__global__ void k(float* out, int iters)
{
    __shared__ uint32_t tptr;
    __shared__ __align__(16) uint32_t stage[16][32 * 64];
    const int warp = threadIdx.x / 32;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tptr)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t base = tptr + ((uint32_t)((warp % 4) * 32) << 16) + (warp / 4) % 4 * 128;
    float acc = 0.f;
    for (int it = 0; it < iters; ++it) {
        uint32_t x[128];
        if (MODE != 2) {
#pragma unroll
            for (int c = 0; c < 4; ++c) ld32(base + c * 32, *reinterpret_cast<uint32_t(*)[32]>(&x[c * 32]));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        } else {
#pragma unroll
            for (int c = 0; c < 128; ++c) x[c] = (uint32_t)(it + c) | 0xbf000000u;
        }
        if (MODE == 3) {
            float m8[8];
#pragma unroll
            for (int a = 0; a < 8; ++a) m8[a] = __uint_as_float(x[a]);
#pragma unroll
            for (int u = 8; u < 128; ++u) m8[u & 7] = fmaxf(m8[u & 7], __uint_as_float(x[u]));
            const float mx = fmaxf(fmaxf(fmaxf(m8[0], m8[1]), fmaxf(m8[2], m8[3])), fmaxf(fmaxf(m8[4], m8[5]), fmaxf(m8[6], m8[7])));
            const float neg = -mx * 0.125f;
#pragma unroll
            for (int u = 0; u < 128; u += 2) {
                float t0, t1;
                t0 = __uint_as_float(x[u]); t1 = __uint_as_float(x[u + 1]);
                ffma2(t0, t1, 0.125f, neg);
                x[u] = __float_as_uint(ex2(t0));
                x[u + 1] = __float_as_uint(ex2(t1));
            }
            float sa[8] = {};
#pragma unroll
            for (int u = 0; u < 128; u += 2) fadd2(sa[(u >> 1) & 3], sa[4 + ((u >> 1) & 3)], __uint_as_float(x[u]), __uint_as_float(x[u + 1]));
            acc += ((sa[0] + sa[4]) + (sa[1] + sa[5])) + ((sa[2] + sa[6]) + (sa[3] + sa[7]));
            uint32_t* st = &stage[warp][0];
#pragma unroll
            for (int q4 = 0; q4 < 16; ++q4) {
                uint4 w;
                w.x = pk(__uint_as_float(x[q4 * 8]), __uint_as_float(x[q4 * 8 + 1]));
                w.y = pk(__uint_as_float(x[q4 * 8 + 2]), __uint_as_float(x[q4 * 8 + 3]));
                w.z = pk(__uint_as_float(x[q4 * 8 + 4]), __uint_as_float(x[q4 * 8 + 5]));
                w.w = pk(__uint_as_float(x[q4 * 8 + 6]), __uint_as_float(x[q4 * 8 + 7]));
                const int lane = threadIdx.x % 32;
                *reinterpret_cast<uint4*>(st + ((q4 >> 3) * 32 * 32 + lane * 32 + (((q4 & 7) ^ (lane & 7)) << 2))) = w;
            }
            __syncwarp();
        } else if (MODE != 0) {
#pragma unroll
            for (int c = 0; c < 128; ++c) acc += ex2(__uint_as_float(x[c] | 0x80000000u) * 1e-30f);
        } else {
#pragma unroll
            for (int c = 0; c < 128; ++c) acc += __uint_as_float(x[c]);
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tptr) : "memory");
}

int main()
{
    int sms, clk;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    float* out;
    cudaMalloc(&out, sms * 1024 * 4);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int iters = 2048;
    const char* names[] = {"tcgen05.ld 32x32b (128 cols)", "ld + 128 ex2", "128 ex2 only", "ld + full LS math + sts"};
    for (int m = 0; m < 4; ++m)
        for (int warps : {4, 8, 12, 16}) {
            float ms = 0;
            for (int rep = 0; rep < 2; ++rep) {
                cudaEventRecord(a);
                if (m == 0) k<0><<<sms, warps * 32>>>(out, iters);
                if (m == 1) k<1><<<sms, warps * 32>>>(out, iters);
                if (m == 2) k<2><<<sms, warps * 32>>>(out, iters);
                if (m == 3) k<3><<<sms, warps * 32>>>(out, iters);
                cudaEventRecord(b);
                cudaEventSynchronize(b);
                cudaEventElapsedTime(&ms, a, b);
            }
            const double cyc = ms * 1e-3 * clk * 1e3;
            const double bytes_per_sm = (double)warps * iters * 32 * 128 * 4;
            printf("%-30s warps %2d: %7.3f ms  %6.1f TMEM B/clk/SM  %6.2f elem/clk/SM  (%.0f clk per 128x128 fp32 tile)\n",
                   names[m], warps, ms, m == 2 ? 0.0 : bytes_per_sm / cyc, bytes_per_sm / 4 / cyc,
                   cyc / ((double)warps * iters / 4));
        }
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
