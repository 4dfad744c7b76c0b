// k_ir.cu -- the IR (inter-sub-vector reduction) sub-layer.
//
// Per query row:  m = max_k m'_k,   d = sum_k e^{m'_k - m} d'_k,   r'_k = e^{m'_k - m} / d.
// The statistics are stored [slot][128 rows].  The kernel moves 8 bytes in + 4 bytes out per (row,
// tile) -- 1/T of the attention-matrix traffic.  The paper keeps IR standalone because
// its GEMM1 thread blocks each own one output tile; this is that layout (variant SR_IR_KERNEL).  The
// default path instead merges the statistics inside GEMM1, whose CTAs own whole rows (R24).
#include "ptx.cuh"
#include "sr_internal.h"

namespace sr {

// Organisation (vectorised): one CTA of kW warps per (head, row-block).  A thread owns 4
// consecutive rows (lane l: rows 4l .. 4l+3, all in one 64-row half), so one warp-wide 16-B load
// (LDG.128) brings a whole tile's 128 statistics -- one 512-B run of the [slot][128] layout.  Warp w
// takes the row-block's tiles w, w + kW, ...: its first kReg tiles' m' stay in registers for the
// r' pass; further tiles are folded 4 at a time (one max, 5 exponentials per row per 4 tiles).  The
// kW partial (m, d) of each row are merged through shared memory, then each warp writes r' for its
// own tiles (re-reading m' beyond the first kReg from L1/L2).  About 15 thread-instructions per
// (row, tile) merge; the kernel moves 12 B per (row, tile).
constexpr int kReg = 4;

__device__ __forceinline__ float4 ldg4(const float* p) { return __ldg(reinterpret_cast<const float4*>(p)); }

template <int kW>
__global__ void __launch_bounds__(kW * 32) ir_kernel(const Params p)
{
    __shared__ float4 part_m[kW][32], part_d[kW][32];
    ptx::griddep_launch_dependents();  // PDL: GEMM2's prologue may start now ...
    ptx::griddep_wait();               // ... and GEMM1's m', d' must be complete before we read them
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int g = blockIdx.x / p.sc.n_rb, rb = blockIdx.x % p.sc.n_rb;
    const int hbit = 16 + (lane >> 4);  // this thread's rows' half-valid bit in the tile info word
    const DevSched& sc = p.sc;
    const int32_t* tp = sc.tp + (size_t)lh_of(sc, g, p.H) * (sc.n_rb + 1);
    const int t0 = __ldg(tp + rb), t1 = __ldg(tp + rb + 1), base = __ldg(tp);
    const int n = t1 - t0;
    // pointers at this warp's first tile (t0 + warp); its k-th tile is at + k * kW * 128 floats
    const int64_t s0 = ((int64_t)g * sc.slots_per_head - base + t0 + warp) * kRowBlock + 4 * lane;
    const float* mp = p.mprime + s0;
    const float* dp = p.dprime + s0;
    float* rp = p.rprime + s0;
    const int32_t* ti = sc.tinfo + t0 + warp;
    const int nw = n > warp ? (n - warp + kW - 1) / kW : 0;  // tiles of this warp
    const float l2e = 1.4426950408889634f;
    constexpr int ST = kW * kRowBlock;

    // base-2 m' of one tile for this thread's 4 rows (-inf on an invalid half: its statistics were
    // never written), and d' (0 there)
    auto load = [&](int u, float (&m4)[4], float (&d4)[4], bool with_d) {
        const bool in = u < nw;
        const bool v = in && ((__ldg(ti + u * kW) >> hbit) & 1);
        float4 mm = make_float4(0.f, 0.f, 0.f, 0.f), dd = mm;
        if (v) {
            mm = ldg4(mp + (int64_t)u * ST);
            if (with_d) dd = ldg4(dp + (int64_t)u * ST);
        }
        m4[0] = v ? mm.x * l2e : -INFINITY; m4[1] = v ? mm.y * l2e : -INFINITY;
        m4[2] = v ? mm.z * l2e : -INFINITY; m4[3] = v ? mm.w * l2e : -INFINITY;
        d4[0] = dd.x; d4[1] = dd.y; d4[2] = dd.z; d4[3] = dd.w;
    };
    float mk[kReg][4], dk[kReg][4];  // [tile][row]
#pragma unroll
    for (int u = 0; u < kReg; ++u) load(u, mk[u], dk[u], true);
    float m[4], d[4];
#pragma unroll
    for (int r = 0; r < 4; ++r) {
        m[r] = fmaxf(fmaxf(mk[0][r], mk[1][r]), fmaxf(mk[2][r], mk[3][r]));
        const float ms = m[r] == -INFINITY ? 0.f : m[r];
        float acc = 0.f;
#pragma unroll
        for (int u = 0; u < kReg; ++u) acc = fmaf(dk[u][r], ptx::ex2(mk[u][r] - ms), acc);
        d[r] = acc;
    }
    for (int tb = kReg; tb < nw; tb += 4) {  // rows longer than kW * kReg tiles
        float m4[4][4], d4[4][4];
#pragma unroll
        for (int u = 0; u < 4; ++u) load(tb + u, m4[u], d4[u], true);
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            const float mn = fmaxf(fmaxf(m[r], fmaxf(m4[0][r], m4[1][r])), fmaxf(m4[2][r], m4[3][r]));
            if (mn == -INFINITY) continue;
            float acc = d[r] * ptx::ex2(m[r] - mn);  // ex2(-inf) = 0 while nothing was seen yet
#pragma unroll
            for (int u = 0; u < 4; ++u) acc = fmaf(d4[u][r], ptx::ex2(m4[u][r] - mn), acc);
            m[r] = mn;
            d[r] = acc;
        }
    }
    // merge the kW partial (m, d) of each row: m = max_w m_w, d = sum_w 2^{m_w - m} d_w
    part_m[warp][lane] = make_float4(m[0], m[1], m[2], m[3]);
    part_d[warp][lane] = make_float4(d[0], d[1], d[2], d[3]);
    __syncthreads();
    float mneg[4], inv_d[4];
    {
        float M[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY}, D[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int w = 0; w < kW; ++w) {
            const float4 pm = part_m[w][lane];
            M[0] = fmaxf(M[0], pm.x); M[1] = fmaxf(M[1], pm.y); M[2] = fmaxf(M[2], pm.z); M[3] = fmaxf(M[3], pm.w);
        }
#pragma unroll
        for (int r = 0; r < 4; ++r) mneg[r] = M[r] == -INFINITY ? 0.f : -M[r];  // all-masked row: terms are 0
#pragma unroll
        for (int w = 0; w < kW; ++w) {
            const float4 pm = part_m[w][lane], pd = part_d[w][lane];
            D[0] = fmaf(pd.x, ptx::ex2(pm.x + mneg[0]), D[0]);
            D[1] = fmaf(pd.y, ptx::ex2(pm.y + mneg[1]), D[1]);
            D[2] = fmaf(pd.z, ptx::ex2(pm.z + mneg[2]), D[2]);
            D[3] = fmaf(pd.w, ptx::ex2(pm.w + mneg[3]), D[3]);
        }
#pragma unroll
        for (int r = 0; r < 4; ++r) inv_d[r] = D[r] > 0.f ? 1.f / D[r] : 0.f;
    }
    // r'_k = 2^{m'_k - m} / d  (0 for invalid halves and fully masked sub-vectors)
    auto store = [&](int u, const float (&m4)[4]) {
        float4 o;
        o.x = ptx::ex2(m4[0] + mneg[0]) * inv_d[0];
        o.y = ptx::ex2(m4[1] + mneg[1]) * inv_d[1];
        o.z = ptx::ex2(m4[2] + mneg[2]) * inv_d[2];
        o.w = ptx::ex2(m4[3] + mneg[3]) * inv_d[3];
        *reinterpret_cast<float4*>(rp + (int64_t)u * ST) = o;
    };
#pragma unroll
    for (int u = 0; u < kReg; ++u)
        if (u < nw) store(u, mk[u]);
    for (int tb = kReg; tb < nw; tb += 4) {
        float m4[4][4], d4[4][4];
#pragma unroll
        for (int u = 0; u < 4; ++u) load(tb + u, m4[u], d4[u], false);
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (tb + u < nw) store(tb + u, m4[u]);
    }
}

cudaError_t launch_ir(const Params& p, cudaStream_t st, int64_t* nlaunch)
{
    // one CTA per (head, row-block); warps by the mean tile-list length (one register round per warp)
    const int64_t blocks = (int64_t)p.B * p.H * p.sc.n_rb;
    // (the longest list sets the critical path: rows of up to kW * kReg tiles take one round trip)
    const int m = p.sc.mean_rb_tiles, mx = p.sc.max_rb_tiles;
    if (m <= 2 * kReg && mx <= 4 * kReg) return launch_pdl(ir_kernel<2>, dim3((unsigned)blocks), dim3(64), 0, st, nlaunch, p);
    if (m <= 4 * kReg && mx <= 8 * kReg) return launch_pdl(ir_kernel<4>, dim3((unsigned)blocks), dim3(128), 0, st, nlaunch, p);
    return launch_pdl(ir_kernel<8>, dim3((unsigned)blocks), dim3(256), 0, st, nlaunch, p);
}

}  // namespace sr
