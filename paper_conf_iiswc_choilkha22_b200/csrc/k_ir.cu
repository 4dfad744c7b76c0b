// k_ir.cu -- the IR (inter-sub-vector reduction) sub-layer.
//
// Per query row:  m = max_k m'_k,   d = sum_k e^{m'_k - m} d'_k,   r'_k = e^{m'_k - m} / d.
// One thread per row.  The statistics are stored [slot][128 rows], so the 32 threads of a warp
// (32 consecutive rows of one row-block) read and write 128 contiguous bytes per tile: fully
// coalesced.  The kernel is HBM/latency bound: 8 bytes read + 4 bytes written per (row, tile),
// i.e. 1/T of the attention-matrix traffic.  It cannot be fused into GEMM1
// (m, d need every tile of the row) -- the paper's design keeps it standalone.
#include "sr_internal.h"

namespace sr {

__global__ void __launch_bounds__(256) ir_kernel(Params p)
{
    const int64_t row = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t n_rows = (int64_t)p.B * p.H * p.S;
    if (row >= n_rows) return;
    const int g = (int)(row / p.S);
    const int i = (int)(row % p.S);
    const int rb = i / kRowBlock, lane = i % kRowBlock, half = lane / kHalf;
    const DevSched& sc = p.sc;
    const int lh = lh_of(sc, g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    const int t0 = tp[rb], t1 = tp[rb + 1], base = tp[0];
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - base;

    // m and d in one pass: batches of 8 independent (m'_k, d'_k) loads, merged with the running
    // (m, d) -- d is rescaled by e^{m_old - m_new} whenever the running max grows.  Same reduction
    // as PAPER.md L147 (m = max m'_k, d = sum e^{m'_k - m} d'_k), regrouped for memory-level
    // parallelism.
    const float* mp = p.mprime + slot0 * kRowBlock + lane;
    const float* dp = p.dprime + slot0 * kRowBlock + lane;
    float m = -INFINITY, d = 0.f;
    for (int tb = t0; tb < t1; tb += 8) {
        float mk[8], dk[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const int t = tb + u;
            const bool ok = t < t1 && ((tinfo_half(__ldg(sc.tinfo + t)) >> half) & 1);
            mk[u] = ok ? __ldg(mp + (int64_t)t * kRowBlock) : -INFINITY;
            dk[u] = ok ? __ldg(dp + (int64_t)t * kRowBlock) : 0.f;
        }
        float mb = mk[0];
#pragma unroll
        for (int u = 1; u < 8; ++u) mb = fmaxf(mb, mk[u]);
        if (mb == -INFINITY) continue;
        const float mn = fmaxf(m, mb);
        float acc = (m == -INFINITY) ? 0.f : d * __expf(m - mn);
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (mk[u] != -INFINITY) acc += dk[u] * __expf(mk[u] - mn);
        m = mn;
        d = acc;
    }
    const float inv_d = d > 0.f ? 1.f / d : 0.f;
    float* rp = p.rprime + slot0 * kRowBlock + lane;
    for (int tb = t0; tb < t1; tb += 8) {
        float mk[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const int t = tb + u;
            const bool ok = t < t1 && ((tinfo_half(__ldg(sc.tinfo + t)) >> half) & 1);
            mk[u] = ok ? __ldg(mp + (int64_t)t * kRowBlock) : -INFINITY;
        }
#pragma unroll
        for (int u = 0; u < 8; ++u)
            if (tb + u < t1) rp[(int64_t)(tb + u) * kRowBlock] = (mk[u] == -INFINITY) ? 0.f : __expf(mk[u] - m) * inv_d;
    }
}

cudaError_t launch_ir(const Params& p, cudaStream_t st, int64_t* nlaunch)
{
    const int64_t n_rows = (int64_t)p.B * p.H * p.S;
    const int threads = 256;
    const int64_t blocks = (n_rows + threads - 1) / threads;
    ir_kernel<<<(unsigned)blocks, threads, 0, st>>>(p);
    ++*nlaunch;
    return cudaGetLastError();
}

}  // namespace sr
