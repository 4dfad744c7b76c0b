// k_ir.cu -- the IR (inter-sub-vector reduction) sub-layer.
//
// Per query row:  m = max_k m'_k,   d = sum_k e^{m'_k - m} d'_k,   r'_k = e^{m'_k - m} / d.
// The statistics are stored [slot][128 rows].  The kernel moves 8 bytes in + 4 bytes out per (row,
// tile) -- 1/T of the attention-matrix traffic -- and is latency-bound, so the loads
// of a row are spread over warps and all issued at once.  It cannot be fused into GEMM1 (m and d need
// every tile of the row); the paper keeps it standalone and so does this design.
#include "ptx.cuh"
#include "sr_internal.h"

namespace sr {

// Organisation: one CTA of kW warps per 32 rows of a row-block (lane = row, so every warp-wide load
// or store is one coalesced 128-B line of a tile's statistics).  The row-block's tile list is split
// round-robin over the warps: warp w takes tiles w, w + kW, ..., holding up to kReg of them in
// registers, so a row of up to kW * kReg tiles costs one round trip to memory; the per-warp partial
// (m, d) pairs are merged through shared memory, and each warp writes r' for its own tiles.
// kW = 2, 4 or 8 by the schedule's mean row length (enough warps for one round trip, no more).
constexpr int kReg = 4;

template <int kW>
__global__ void __launch_bounds__(kW * 32) ir_kernel(const Params p)
{
    __shared__ float part_m[kW][32], part_d[kW][32];
    ptx::griddep_launch_dependents();  // PDL: GEMM2's prologue may start now ...
    ptx::griddep_wait();               // ... and GEMM1's m', d' must be complete before we read them
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int64_t row0 = (int64_t)blockIdx.x * 32;  // 32 rows of one row-block (S % 128 == 0)
    const int g = (int)(row0 / p.S);
    const int i0 = (int)(row0 % p.S);
    const int rb = i0 / kRowBlock, r = i0 % kRowBlock + lane;
    const int hbit = 16 + r / kHalf;  // this row's half-valid bit in the tile info word
    const DevSched& sc = p.sc;
    const int32_t* tp = sc.tp + (size_t)lh_of(sc, g, p.H) * (sc.n_rb + 1);
    const int t0 = __ldg(tp + rb), t1 = __ldg(tp + rb + 1), base = __ldg(tp);
    const int n = t1 - t0;
    // pointers at this warp's first tile (t0 + warp); its k-th tile is at + k * kW * 128 floats
    const int64_t s0 = ((int64_t)g * sc.slots_per_head - base + t0 + warp) * kRowBlock + r;
    const float* mp = p.mprime + s0;
    const float* dp = p.dprime + s0;
    float* rp = p.rprime + s0;
    const int32_t* ti = sc.tinfo + t0 + warp;
    const int nw = n > warp ? (n - warp + kW - 1) / kW : 0;  // tiles of this warp
    const float l2e = 1.4426950408889634f;
    constexpr int ST = kW * kRowBlock;

    // one round trip: tile info, m'_k and d'_k of the warp's first kReg tiles (statistics of an
    // invalid 64-row half were never written and are masked out here)
    float mk[kReg], dk[kReg];
#pragma unroll
    for (int u = 0; u < kReg; ++u) {
        const bool in = u < nw;
        const int w = in ? __ldg(ti + u * kW) : 0;
        const float m_ = in ? __ldg(mp + u * ST) : 0.f;
        const float d_ = in ? __ldg(dp + u * ST) : 0.f;
        const bool v = (w >> hbit) & 1;
        mk[u] = v ? m_ * l2e : -INFINITY;  // base 2 from here on
        dk[u] = v ? d_ : 0.f;
    }
    float m = -INFINITY;
#pragma unroll
    for (int u = 0; u < kReg; ++u) m = fmaxf(m, mk[u]);
    float d = 0.f;
#pragma unroll
    for (int u = 0; u < kReg; ++u) d = fmaf(dk[u], ptx::ex2(mk[u] - (m == -INFINITY ? 0.f : m)), d);
    // tiles beyond kReg per warp (rows longer than kW * kReg tiles): fold in 4 at a time
    for (int tb = kReg; tb < nw; tb += 4) {
        float m4[4], d4[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const bool in = tb + u < nw;
            const int w = in ? __ldg(ti + (tb + u) * kW) : 0;
            const float m_ = in ? __ldg(mp + (tb + u) * ST) : 0.f;
            const float d_ = in ? __ldg(dp + (tb + u) * ST) : 0.f;
            m4[u] = ((w >> hbit) & 1) ? m_ * l2e : -INFINITY;
            d4[u] = ((w >> hbit) & 1) ? d_ : 0.f;
        }
        const float mn = fmaxf(fmaxf(m, fmaxf(m4[0], m4[1])), fmaxf(m4[2], m4[3]));
        if (mn == -INFINITY) continue;
        float acc = d * ptx::ex2(m - mn);  // ex2(-inf) = 0 while nothing was seen yet
#pragma unroll
        for (int u = 0; u < 4; ++u) acc = fmaf(d4[u], ptx::ex2(m4[u] - mn), acc);
        m = mn;
        d = acc;
    }
    // merge the kW partial (m, d) of each row: m = max_w m_w, d = sum_w 2^{m_w - m} d_w
    part_m[warp][lane] = m;
    part_d[warp][lane] = d;
    __syncthreads();
    float M = -INFINITY;
#pragma unroll
    for (int w = 0; w < kW; ++w) M = fmaxf(M, part_m[w][lane]);
    const float mneg = M == -INFINITY ? 0.f : -M;  // all-masked row: every term below is 0
    float D = 0.f;
#pragma unroll
    for (int w = 0; w < kW; ++w) D = fmaf(part_d[w][lane], ptx::ex2(part_m[w][lane] + mneg), D);
    const float inv_d = D > 0.f ? 1.f / D : 0.f;
    // r'_k = 2^{m'_k - m} / d  (0 for invalid halves and fully masked sub-vectors)
#pragma unroll
    for (int u = 0; u < kReg; ++u)
        if (u < nw) rp[u * ST] = ptx::ex2(mk[u] + mneg) * inv_d;
    for (int tb = kReg; tb < nw; tb += 4) {
        float m4[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const bool in = tb + u < nw;
            const int w = in ? __ldg(ti + (tb + u) * kW) : 0;
            const float m_ = in ? __ldg(mp + (tb + u) * ST) : 0.f;
            m4[u] = ((w >> hbit) & 1) ? m_ * l2e : -INFINITY;
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (tb + u < nw) rp[(tb + u) * ST] = ptx::ex2(m4[u] + mneg) * inv_d;
    }
}

cudaError_t launch_ir(const Params& p, cudaStream_t st, int64_t* nlaunch)
{
    const int64_t blocks = (int64_t)p.B * p.H * p.S / 32;
    const int m = p.sc.mean_rb_tiles;
    if (m <= kReg) return launch_pdl(ir_kernel<2>, dim3((unsigned)blocks), dim3(64), 0, st, nlaunch, p);
    if (m <= 3 * kReg) return launch_pdl(ir_kernel<4>, dim3((unsigned)blocks), dim3(128), 0, st, nlaunch, p);
    return launch_pdl(ir_kernel<8>, dim3((unsigned)blocks), dim3(256), 0, st, nlaunch, p);
}

}  // namespace sr
