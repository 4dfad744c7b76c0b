// Throughput microbenchmark of the epilogue's instruction mix on one B200:
// MUFU.EX2, F2FP (cvt.rn.f16x2.f32), FFMA2, FMNMX, and a software exp2 (FMA-pipe polynomial).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ub/sfu tools/ubench_sfu.cu && /tmp/ub/sfu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__device__ __forceinline__ unsigned pk(float a, float b) { unsigned r; asm volatile("cvt.rn.f16x2.f32 %0, %2, %1;" : "=r"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ void ffma2(float& a, float& b, float s, float c)
{
    unsigned long long x = ((unsigned long long)__float_as_uint(b) << 32) | __float_as_uint(a);
    unsigned long long sc = ((unsigned long long)__float_as_uint(s) << 32) | __float_as_uint(s);
    unsigned long long cc = ((unsigned long long)__float_as_uint(c) << 32) | __float_as_uint(c);
    asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(x) : "l"(sc), "l"(cc));
    a = __uint_as_float((unsigned)x); b = __uint_as_float((unsigned)(x >> 32));
}
// software 2^t for t <= 0: round-to-nearest split, degree-3 polynomial on [-0.5, 0.5]
__device__ __forceinline__ float sw_ex2(float t)
{
    t = fmaxf(t, -127.f);
    const float r = t + 12582912.f;
    const float j = r - 12582912.f;
    const float f = t - j;
    float p = fmaf(f, 0.055171666814681324f, 0.24261113509452378f);  // minimax, rel. err 7.5e-5
    p = fmaf(p, f, 0.6932609870112002f);
    p = fmaf(p, f, 0.9999280727914261f);
    return __uint_as_float(__float_as_uint(p) + (__float_as_uint(r) << 23));
}

template <int MODE>
__global__ void k(float* out, int iters, float s)
{
    float v[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = -(threadIdx.x + i) * 1e-3f;
    unsigned acc = 0;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 16; i += 2) {
            if (MODE == 0) { v[i] = ex2(v[i]) - 1.f; v[i + 1] = ex2(v[i + 1]) - 1.f; }
            if (MODE == 1) { acc ^= pk(v[i], v[i + 1]); v[i] += s; }
            if (MODE == 2) { ffma2(v[i], v[i + 1], s, -1e-3f); }
            if (MODE == 3) { v[i] = ex2(v[i]) - 1.f; v[i + 1] = ex2(v[i + 1]) - 1.f; acc ^= pk(v[i], v[i + 1]); }
            if (MODE == 4) { v[i] = sw_ex2(v[i]) - 1.f; v[i + 1] = sw_ex2(v[i + 1]) - 1.f; }
        }
    }
    float t = 0;
#pragma unroll
    for (int i = 0; i < 16; ++i) t += v[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = t + acc;
}

int main()
{
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    float* out; cudaMalloc(&out, sms * 8 * 1024 * 4);
    const char* names[] = {"MUFU.EX2 (elem)", "F2FP pack (pairs)", "FFMA2 (pairs)", "EX2+F2FP (elem)", "sw exp2 deg3 (elem)"};
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    const int iters = 4096;
    for (int m = 0; m < 5; ++m) {
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(a);
            switch (m) {
            case 0: k<0><<<sms * 4, 512>>>(out, iters, 1e-3f); break;
            case 1: k<1><<<sms * 4, 512>>>(out, iters, 1e-3f); break;
            case 2: k<2><<<sms * 4, 512>>>(out, iters, 1e-3f); break;
            case 3: k<3><<<sms * 4, 512>>>(out, iters, 1e-3f); break;
            case 4: k<4><<<sms * 4, 512>>>(out, iters, 1e-3f); break;
            }
            cudaEventRecord(b); cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            double ops = (double)sms * 4 * 512 * iters * (m == 1 || m == 2 ? 8 : 16);
            if (rep) printf("%-22s %8.3f ms  %7.2f per clk per SM (at %d MHz nominal)\n", names[m], ms,
                            ops / (ms * 1e-3) / sms / (clk * 1e3), clk / 1000);
        }
    }
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
