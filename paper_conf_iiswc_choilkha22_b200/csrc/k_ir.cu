// k_ir.cu -- the IR (inter-sub-vector reduction) sub-layer.
//
// Per query row:  m = max_k m'_k,   d = sum_k e^{m'_k - m} d'_k,   r'_k = e^{m'_k - m} / d.
// One thread per row.  The statistics are stored [slot][128 rows], so the 32 threads of a warp
// (32 consecutive rows of one row-block) read and write 128 contiguous bytes per tile: fully
// coalesced.  The kernel moves 8 bytes in + 4 bytes out per (row, tile) -- 1/T of the
// attention-matrix traffic -- and is latency-bound, so every load of a row is
// issued at once: up to kReg tiles are held in registers (one round trip to memory, then r' from
// registers); longer rows stream the rest in batches.  It cannot be fused into GEMM1 (m and d need
// every tile of the row); the paper keeps it standalone and so does this design.
#include "ptx.cuh"
#include "sr_internal.h"

namespace sr {

constexpr int kReg = 16;

__global__ void __launch_bounds__(256) ir_kernel(const Params p)
{
    ptx::griddep_launch_dependents();  // PDL: GEMM2's prologue may start now ...
    ptx::griddep_wait();               // ... and GEMM1's m', d' must be complete before we read them
    const int64_t row = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t n_rows = (int64_t)p.B * p.H * p.S;
    if (row >= n_rows) return;
    const int g = (int)(row / p.S);
    const int i = (int)(row % p.S);
    const int rb = i / kRowBlock, lane = i % kRowBlock, half = lane / kHalf;
    const DevSched& sc = p.sc;
    const int lh = lh_of(sc, g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    const int t0 = __ldg(tp + rb), t1 = __ldg(tp + rb + 1), base = __ldg(tp);
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - base;
    const float* mp = p.mprime + slot0 * kRowBlock + lane;
    const float* dp = p.dprime + slot0 * kRowBlock + lane;
    float* rp = p.rprime + slot0 * kRowBlock + lane;

    // round trip 1: tile info, m'_k and d'_k of the first kReg tiles, all independent loads (the
    // statistics of an invalid 64-row half were never written and are masked out afterwards)
    float mk[kReg], dk[kReg];
    bool ok[kReg];
#pragma unroll
    for (int u = 0; u < kReg; ++u) {
        const int t = t0 + u;
        const bool in = t < t1;
        const int w = in ? __ldg(sc.tinfo + t) : 0;
        const float m_ = in ? __ldg(mp + (int64_t)t * kRowBlock) : -INFINITY;
        const float d_ = in ? __ldg(dp + (int64_t)t * kRowBlock) : 0.f;
        ok[u] = in && ((tinfo_half(w) >> half) & 1);
        mk[u] = ok[u] ? m_ : -INFINITY;
        dk[u] = ok[u] ? d_ : 0.f;
    }
    float m = -INFINITY;
#pragma unroll
    for (int u = 0; u < kReg; ++u) m = fmaxf(m, mk[u]);
    // tiles beyond kReg (rows longer than kReg * T keys): fold into a running (m, d)
    float d_tail = 0.f;
    for (int tb = t0 + kReg; tb < t1; tb += 8) {
        float m8[8], d8[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const int t = tb + u;
            const bool in = t < t1;
            const int w = in ? __ldg(sc.tinfo + t) : 0;
            const float m_ = in ? __ldg(mp + (int64_t)t * kRowBlock) : -INFINITY;
            const float d_ = in ? __ldg(dp + (int64_t)t * kRowBlock) : 0.f;
            const bool v = in && ((tinfo_half(w) >> half) & 1);
            m8[u] = v ? m_ : -INFINITY;
            d8[u] = v ? d_ : 0.f;
        }
        float mb = m8[0];
#pragma unroll
        for (int u = 1; u < 8; ++u) mb = fmaxf(mb, m8[u]);
        if (mb == -INFINITY) continue;
        const float mn = fmaxf(m, mb);
        float acc = (m == -INFINITY) ? 0.f : d_tail * __expf(m - mn);
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (m8[u] != -INFINITY) acc += d8[u] * __expf(m8[u] - mn);
        m = mn;
        d_tail = acc;
    }
    // d = sum_k e^{m'_k - m} d'_k
    float d = d_tail;
#pragma unroll
    for (int u = 0; u < kReg; ++u)
        if (mk[u] != -INFINITY) d += dk[u] * __expf(mk[u] - m);
    const float inv_d = d > 0.f ? 1.f / d : 0.f;
    // r'_k = e^{m'_k - m} / d  (0 for invalid halves and fully masked sub-vectors)
#pragma unroll
    for (int u = 0; u < kReg; ++u)
        if (t0 + u < t1) rp[(int64_t)(t0 + u) * kRowBlock] = (mk[u] == -INFINITY) ? 0.f : __expf(mk[u] - m) * inv_d;
    for (int t = t0 + kReg; t < t1; ++t) {
        const int w = __ldg(sc.tinfo + t);
        const float m_ = __ldg(mp + (int64_t)t * kRowBlock);
        const bool v = (tinfo_half(w) >> half) & 1;
        rp[(int64_t)t * kRowBlock] = (!v || m_ == -INFINITY) ? 0.f : __expf(m_ - m) * inv_d;
    }
}

cudaError_t launch_ir(const Params& p, cudaStream_t st, int64_t* nlaunch)
{
    const int64_t n_rows = (int64_t)p.B * p.H * p.S;
    const int threads = 256;
    const int64_t blocks = (n_rows + threads - 1) / threads;
    return launch_pdl(ir_kernel, dim3((unsigned)blocks), dim3(threads), 0, st, nlaunch, p);
}

}  // namespace sr
