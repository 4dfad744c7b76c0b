// k_simt_f32.cu -- fp32 mode of the recomposed chain (BASELINE config 1, tolerance 1e-5).
//
// Same three-kernel structure as the tensor-core path (GEMM1+LS -> IR -> GS+GEMM2, PAPER.md
// L165), on CUDA cores with FFMA: kind::tf32 tensor cores would give ~6.6e-4 error (SURVEY
// App. A.4), above the 1e-5 fp32 tolerance of the north star.  One CTA per item (head, 128-row
// block), one thread per query row, T = 64.  X' is stored fp32 row-major [128][64] per slot.
#include "sr_internal.h"

namespace sr {

template <int D>
__global__ void __launch_bounds__(128) simt_gemm1_ls_f32(Params p)
{
    extern __shared__ float ks[];  // K tile [64][D]
    constexpr int T = 64;
    const DevSched& sc = p.sc;
    const int item = sc.items[blockIdx.x];
    const int g = item / sc.n_rb, rb = item % sc.n_rb;
    const int lh = lh_of(sc, g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    const int t0 = tp[rb], t1 = tp[rb + 1];
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - tp[0];
    const int tid = threadIdx.x, i = rb * kRowBlock + tid;
    const int kvl = sc.kv_len ? sc.kv_len[g / p.H] : p.S;
    const float* Q = (const float*)p.q + ((size_t)g * p.S + i) * D;
    const float* K = (const float*)p.k + (size_t)g * p.S * D;
    float q[D];
#pragma unroll
    for (int d = 0; d < D; ++d) q[d] = i < p.S ? Q[d] : 0.f;  // rows beyond the head (S % 128 == 64): invalid half

    for (int t = t0; t < t1; ++t) {
        const int w = sc.tinfo[t], kt = tinfo_kt(w);
        __syncthreads();
        for (int e = tid; e < T * D; e += blockDim.x) ks[e] = K[(size_t)kt * T * D + e];
        __syncthreads();
        if (!((tinfo_half(w) >> (tid / kHalf)) & 1)) continue;
        // LS: scores of this row's sub-vector, local max m', X' = e^{x - m'}, local sum d'
        float x[T];
        float m = -INFINITY;
#pragma unroll 4
        for (int c = 0; c < T; ++c) {
            const float* kr = ks + c * D;
            float s = 0.f;
#pragma unroll
            for (int d = 0; d < D; ++d) s = fmaf(q[d], kr[d], s);
            const int j = kt * T + c;
            x[c] = elem_kept(p, kvl, i, j) ? s * p.scale : -INFINITY;
            m = fmaxf(m, x[c]);
        }
        float* X = (float*)p.xprime + ((slot0 + t) * kRowBlock + tid) * T;
        float dsum = 0.f;
#pragma unroll 4
        for (int c = 0; c < T; ++c) {
            const float e = (x[c] == -INFINITY) ? 0.f : expf(x[c] - m);
            X[c] = e;
            dsum += e;
        }
        p.mprime[(slot0 + t) * kRowBlock + tid] = m;
        p.dprime[(slot0 + t) * kRowBlock + tid] = dsum;
    }
}

template <int D>
__global__ void __launch_bounds__(128) simt_gs_gemm2_f32(Params p)
{
    extern __shared__ float sm[];
    constexpr int T = 64, XS = T + 1;  // X' row stride padded against bank conflicts
    float* vs = sm;                    // V tile [64][D]
    float* xs = sm + T * D;            // X' tile [128][65]
    const DevSched& sc = p.sc;
    const int item = sc.items[blockIdx.x];
    const int g = item / sc.n_rb, rb = item % sc.n_rb;
    const int lh = lh_of(sc, g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    const int t0 = tp[rb], t1 = tp[rb + 1];
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - tp[0];
    const int tid = threadIdx.x, i = rb * kRowBlock + tid;
    const float* V = (const float*)p.v + (size_t)g * p.S * D;
    float o[D];
#pragma unroll
    for (int d = 0; d < D; ++d) o[d] = 0.f;

    for (int t = t0; t < t1; ++t) {
        const int w = sc.tinfo[t], kt = tinfo_kt(w);
        __syncthreads();
        for (int e = tid; e < T * D; e += blockDim.x) vs[e] = V[(size_t)kt * T * D + e];
        const float* X = (const float*)p.xprime + (slot0 + t) * kRowBlock * T;
        for (int e = tid; e < kRowBlock * T; e += blockDim.x) xs[(e / T) * XS + e % T] = X[e];
        __syncthreads();
        // GS: y = X' * r'  (r' = 0 for an invalid half or a fully masked sub-vector)
        const float r = ((tinfo_half(w) >> (tid / kHalf)) & 1) ? p.rprime[(slot0 + t) * kRowBlock + tid] : 0.f;
        if (r == 0.f) continue;
        for (int c = 0; c < T; ++c) {
            const float y = xs[tid * XS + c] * r;
            const float* vr = vs + c * D;
#pragma unroll
            for (int d = 0; d < D; ++d) o[d] = fmaf(y, vr[d], o[d]);
        }
    }
    if (i >= p.S) return;  // a row beyond the head (S % 128 == 64)
    float* O = (float*)p.out + ((size_t)g * p.S + i) * D;
#pragma unroll
    for (int d = 0; d < D; ++d) O[d] = o[d];
}

template <int D>
static cudaError_t launch_d(const Params& p, cudaStream_t st, int64_t* nl)
{
    const int n = p.sc.n_items;
    size_t sm1 = 64 * D * sizeof(float);
    size_t sm2 = (64 * D + kRowBlock * 65) * sizeof(float);
    cudaError_t e = cudaFuncSetAttribute(simt_gemm1_ls_f32<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm1);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(simt_gs_gemm2_f32<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm2);
    if (e != cudaSuccess) return e;
    if (p.stages & 1) {
        simt_gemm1_ls_f32<D><<<n, 128, sm1, st>>>(p);
        ++*nl;
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    if ((p.stages & 2) && (e = launch_ir(p, st, nl)) != cudaSuccess) return e;
    if (p.stages & 4) {
        simt_gs_gemm2_f32<D><<<n, 128, sm2, st>>>(p);
        ++*nl;
        e = cudaGetLastError();
    }
    return e;
}

cudaError_t launch_simt_f32(const Params& p, cudaStream_t st, int64_t* nl)
{
    return p.D == 64 ? launch_d<64>(p, st, nl) : launch_d<128>(p, st, nl);
}

}  // namespace sr
