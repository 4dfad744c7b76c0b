// k_simt_f32.cu -- fp32 mode of the recomposed chain (BASELINE config 1, tolerance 1e-5).
//
// Same three-kernel structure as the tensor-core path (GEMM1+LS -> IR -> GS+GEMM2, PAPER.md
// L165), on CUDA cores with FFMA: kind::tf32 tensor cores would give ~6.6e-4 error (SURVEY
// App. A.4), above the 1e-5 fp32 tolerance of the north star.  T = 64; X' is stored fp32 row-major
// [128][64] per slot.  A CTA takes 128 / TPR rows of an item (head, 128-row block), so a
// 64-row half -- the validity granularity -- is uniform per CTA; TPR threads share a row: in
// GEMM1 thread c owns the tile's columns c, c + TPR, ... (K rows padded to D + 1 floats: the
// threads of a row read distinct banks), max and sum meet by shuffles; in GEMM2 thread c owns output
// columns c, c + TPR, ...  TPR (4, 8, 16 or 32) is the smallest that gives >= 2 CTAs per
// SM, else 32 (few items: C1, one 128-row block, round 1's one CTA with a thread per row walking 64
// columns x D serially took 82.4 us per layer, 4 threads per row 35.1, 16 19.7, 32 16.7 us; with
// many items 4 is fastest -- B1 H12 S2048 D64 causal: 812 / 866 / 1019 us at 4 / 16 / 32).
#include "sr_internal.h"

namespace sr {


template <int D, int TPR>
__global__ void __launch_bounds__(128) simt_gemm1_ls_f32(Params p)
{
    constexpr int ROWS = 128 / TPR;  // rows per CTA
    extern __shared__ float ks[];  // K tile [64][D + 1]
    constexpr int T = 64, KS = D + 1, NC = T / TPR;
    const DevSched& sc = p.sc;
    const int item = sc.items[blockIdx.x];
    const int g = item / sc.n_rb, rb = item % sc.n_rb;
    const int lh = lh_of(sc, g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    const int t0 = tp[rb], t1 = tp[rb + 1];
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - tp[0];
    const int tid = threadIdx.x, cg = tid % TPR, rr = blockIdx.y * ROWS + tid / TPR, i = rb * kRowBlock + rr;
    const int kvl = sc.kv_len ? sc.kv_len[g / p.H] : p.S;
    const float* Q = (const float*)p.q + ((size_t)g * p.S + i) * D;
    const float* K = (const float*)p.k + (size_t)g * p.S * D;
    float q[D];
#pragma unroll
    for (int d = 0; d < D; ++d) q[d] = i < p.S ? Q[d] : 0.f;  // rows beyond the head (S % 128 == 64): invalid half

    for (int t = t0; t < t1; ++t) {
        const int w = sc.tinfo[t], kt = tinfo_kt(w);
        __syncthreads();
        for (int e = tid; e < T * D; e += blockDim.x) ks[(e / D) * KS + e % D] = K[(size_t)kt * T * D + e];
        __syncthreads();
        if (!((tinfo_half(w) >> (rr / kHalf)) & 1)) continue;  // uniform: the CTA's rows are in one half
        // LS: scores of this row's sub-vector, local max m', X' = e^{x - m'}, local sum d'
        float x[NC];
#pragma unroll
        for (int j = 0; j < NC; ++j) x[j] = 0.f;
#pragma unroll
        for (int d = 0; d < D; ++d)
#pragma unroll
            for (int j = 0; j < NC; ++j) x[j] = fmaf(q[d], ks[(cg + TPR * j) * KS + d], x[j]);
        float m = -INFINITY;
#pragma unroll
        for (int j = 0; j < NC; ++j) {
            x[j] = elem_kept(p, kvl, i, kt * T + cg + TPR * j) ? x[j] * p.scale : -INFINITY;
            m = fmaxf(m, x[j]);
        }
#pragma unroll
        for (int o = 1; o < TPR; o <<= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
        float* X = (float*)p.xprime + ((slot0 + t) * kRowBlock + rr) * T;
        float dsum = 0.f;
#pragma unroll
        for (int j = 0; j < NC; ++j) {
            const float e = (x[j] == -INFINITY) ? 0.f : expf(x[j] - m);
            X[cg + TPR * j] = e;
            dsum += e;
        }
#pragma unroll
        for (int o = 1; o < TPR; o <<= 1) dsum += __shfl_xor_sync(0xffffffffu, dsum, o);
        if (cg == 0) {
            p.mprime[(slot0 + t) * kRowBlock + rr] = m;
            p.dprime[(slot0 + t) * kRowBlock + rr] = dsum;
        }
    }
}

template <int D, int TPR>
__global__ void __launch_bounds__(128) simt_gs_gemm2_f32(Params p)
{
    constexpr int ROWS = 128 / TPR;  // rows per CTA
    extern __shared__ float sm[];
    constexpr int T = 64, XS = T + 1, ND = D / TPR;  // X' row stride padded against bank conflicts
    float* vs = sm;                                // V tile [64][D]
    float* xs = sm + T * D;                        // X' rows of this CTA [ROWS][65]
    const DevSched& sc = p.sc;
    const int item = sc.items[blockIdx.x];
    const int g = item / sc.n_rb, rb = item % sc.n_rb;
    const int lh = lh_of(sc, g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    const int t0 = tp[rb], t1 = tp[rb + 1];
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - tp[0];
    const int tid = threadIdx.x, cg = tid % TPR, r = tid / TPR, rr = blockIdx.y * ROWS + r, i = rb * kRowBlock + rr;
    const float* V = (const float*)p.v + (size_t)g * p.S * D;
    float o[ND];
#pragma unroll
    for (int k = 0; k < ND; ++k) o[k] = 0.f;

    for (int t = t0; t < t1; ++t) {
        const int w = sc.tinfo[t], kt = tinfo_kt(w);
        if (!((tinfo_half(w) >> (rr / kHalf)) & 1)) continue;  // uniform per CTA
        __syncthreads();
        for (int e = tid; e < T * D; e += blockDim.x) vs[e] = V[(size_t)kt * T * D + e];
        const float* X = (const float*)p.xprime + ((slot0 + t) * kRowBlock + blockIdx.y * ROWS) * T;
        for (int e = tid; e < ROWS * T; e += blockDim.x) xs[(e / T) * XS + e % T] = X[e];
        __syncthreads();
        // GS: y = X' * r'  (r' = 0 for a fully masked sub-vector)
        const float rf = p.rprime[(slot0 + t) * kRowBlock + rr];
        if (rf == 0.f) continue;
        for (int c = 0; c < T; ++c) {
            const float y = xs[r * XS + c] * rf;
            const float* vr = vs + c * D + cg;
#pragma unroll
            for (int k = 0; k < ND; ++k) o[k] = fmaf(y, vr[TPR * k], o[k]);
        }
    }
    if (i >= p.S) return;  // a row beyond the head (S % 128 == 64)
    float* O = (float*)p.out + ((size_t)g * p.S + i) * D;
#pragma unroll
    for (int k = 0; k < ND; ++k) O[cg + TPR * k] = o[k];
}

template <int D, int TPR>
static cudaError_t launch_d(const Params& p, cudaStream_t st, int64_t* nl)
{
    const dim3 grid(p.sc.n_items, TPR);  // TPR CTAs of 128 / TPR rows per item
    size_t sm1 = 64 * (D + 1) * sizeof(float);
    size_t sm2 = (64 * D + (128 / TPR) * 65) * sizeof(float);
    cudaError_t e = cudaFuncSetAttribute(simt_gemm1_ls_f32<D, TPR>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm1);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(simt_gs_gemm2_f32<D, TPR>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm2);
    if (e != cudaSuccess) return e;
    if (p.stages & 1) {
        simt_gemm1_ls_f32<D, TPR><<<grid, 128, sm1, st>>>(p);
        ++*nl;
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    if ((p.stages & 2) && (e = launch_ir(p, st, nl)) != cudaSuccess) return e;
    if (p.stages & 4) {
        simt_gs_gemm2_f32<D, TPR><<<grid, 128, sm2, st>>>(p);
        ++*nl;
        e = cudaGetLastError();
    }
    return e;
}

template <int D>
static cudaError_t launch_tpr(const Params& p, cudaStream_t st, int64_t* nl)
{
    switch (p.sc.simt_tpr) {  // chosen on the host (make_blob) from the item count
        case 32: return launch_d<D, 32>(p, st, nl);
        case 16: return launch_d<D, 16>(p, st, nl);
        case 8: return launch_d<D, 8>(p, st, nl);
        default: return launch_d<D, 4>(p, st, nl);
    }
}

cudaError_t launch_simt_f32(const Params& p, cudaStream_t st, int64_t* nl)
{
    return p.D == 64 ? launch_tpr<64>(p, st, nl) : launch_tpr<128>(p, st, nl);
}

}  // namespace sr
