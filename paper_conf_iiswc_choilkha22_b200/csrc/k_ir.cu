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

// Organisation (vectorised).  A thread owns 4 consecutive rows of a row-block (lane l: rows 4l ..
// 4l+3, all in one 64-row half), so one warp-wide 16-B load (LDG.128) brings a whole tile's 128
// statistics -- one 512-B run of the [slot][128] layout.  Each row-block gets a TEAM of TW warps
// (TW = 1, 2, 4 or 8, so that a warp has at most KR of its tiles; KR = kIrWarpTiles = 4, or
// kIrWarpTilesWide = 6 when the 4-tile classes would need more than one wave of CTAs -- chosen on the
// host, sc.ir_warp_tiles): warp t of the team
// takes tiles t, t + TW, ..., loads all of them at once (m' and d' in registers: one memory round
// trip), merges them into a partial (m, d) per row; the team's partials meet in shared memory; each
// warp then writes r' for its own tiles.  Row-blocks come longest first (sc.ir_desc) in classes of
// equal TW; a CTA of 8 warps runs 8 / TW row-blocks of one class, and the team size is a template
// parameter (the class is decoded with shifts; the team loops unroll).  Rows longer than 8 * KR
// tiles fold the excess 2 tiles at a time and re-read m'.
// Exponentials: the merge computes e_k = 2^{m'_k - m_w} against the warp's own maximum m_w and keeps
// it, so r'_k = e_k * (2^{m_w - m} / d) costs one multiply per (row, tile) instead of a second
// exponential (the per-row factor is one ex2).  12 B per (row, tile); ncu at C4: 34
// thread-instructions per (row, tile), down from 46 with runtime team sizes and two exponentials.
constexpr int kW = 8;
constexpr int kFold = 2;  // tiles per folding step beyond 8 * KR (register budget)

__device__ __forceinline__ float4 ldg4(const float* p) { return __ldcg(reinterpret_cast<const float4*>(p)); }

// base-2 m' of tile u (pointer offset in tiles) for the thread's 4 rows (-inf on an invalid half:
// its statistics were never written) and d' (0 there)
__device__ __forceinline__ void ir_load(const float* mp, const float* dp, const int32_t* ti, int hbit, int u, bool in,
                                        float (&m4)[4], float (&d4)[4], bool with_d)
{
    const float l2e = 1.4426950408889634f;
    // the statistics are loaded whether or not the half is valid (the slot exists; an invalid half's
    // values are never used), so these loads and the tile word's load share one memory round trip
    float4 mm = make_float4(0.f, 0.f, 0.f, 0.f), dd = mm;
    if (in) {
        mm = ldg4(mp + (int64_t)u * kRowBlock);
        if (with_d) dd = ldg4(dp + (int64_t)u * kRowBlock);
    }
    const bool v = in && ((__ldcg(ti + u) >> hbit) & 1);
    if (!v) dd = make_float4(0.f, 0.f, 0.f, 0.f);
    m4[0] = v ? mm.x * l2e : -INFINITY; m4[1] = v ? mm.y * l2e : -INFINITY;
    m4[2] = v ? mm.z * l2e : -INFINITY; m4[3] = v ? mm.w * l2e : -INFINITY;
    d4[0] = dd.x; d4[1] = dd.y; d4[2] = dd.z; d4[3] = dd.w;
}

// r'_k of tile u = s4 (the thread's 4 rows), 0 for invalid halves and fully masked sub-vectors
__device__ __forceinline__ void ir_store(float* rp, int u, const float (&s4)[4])
{
    *reinterpret_cast<float4*>(rp + (int64_t)u * kRowBlock) = make_float4(s4[0], s4[1], s4[2], s4[3]);
}

#ifndef SR_IR_MIN_CTAS
#define SR_IR_MIN_CTAS 3  // resident CTAs per SM the register budget must allow (see kIrWarpTiles)
#endif

// one team of TW warps per row-block; row-block idx of the class that starts at `first` (nc of them)
template <int TW, int KR>
__device__ __forceinline__ void ir_team(const Params& p, int idx, bool live, float4 (*part_m)[32], float4 (*part_d)[32])
{
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int team = warp / TW, tmw = warp % TW;  // team within the CTA, warp within the team
    const DevSched& sc = p.sc;
    int n = 0;
    const float *mp = nullptr, *dp = nullptr;
    float* rp = nullptr;
    const int32_t* ti = nullptr;
    if (live) {
        const int4 dsc = __ldcg(sc.ir_desc + idx);  // one 16-B load: first slot, tiles, first tile index
        const int64_t s0 = ((int64_t)dsc.x + tmw) * kRowBlock + 4 * lane;
        mp = p.mprime + s0; dp = p.dprime + s0; rp = p.rprime + s0; ti = sc.tinfo + dsc.z + tmw;
        n = dsc.y;
    }
    const int hbit = 16 + (lane >> 4);
    const int nw = n > tmw ? (n - tmw + TW - 1) / TW : 0;  // tiles of this warp: tmw, tmw + TW, ...
    float mk[KR][4], dk[KR][4];  // [tile][row]; mk becomes e_k = 2^{m'_k - m_w}
#pragma unroll
    for (int u = 0; u < KR; ++u) ir_load(mp, dp, ti, hbit, u * TW, u < nw, mk[u], dk[u], true);  // all in flight
    float m[4], d[4], mw[4];  // running (m, d); mw: the maximum the kept e_k are relative to
#pragma unroll
    for (int r = 0; r < 4; ++r) {
        float mx = -INFINITY;
#pragma unroll
        for (int u = 0; u < KR; ++u) mx = fmaxf(mx, mk[u][r]);
        const float ms = mx == -INFINITY ? 0.f : mx;
        float acc = 0.f;
#pragma unroll
        for (int u = 0; u < KR; ++u) {
            mk[u][r] = ptx::ex2(mk[u][r] - ms);  // 0 for -inf
            acc = fmaf(dk[u][r], mk[u][r], acc);
        }
        m[r] = mx;
        mw[r] = mx;
        d[r] = acc;
    }
    for (int tb = KR; tb < nw; tb += kFold) {  // rows longer than 8 * kIrWarpTiles tiles
        float m4[kFold][4], d4[kFold][4];
#pragma unroll
        for (int u = 0; u < kFold; ++u) ir_load(mp, dp, ti, hbit, (tb + u) * TW, tb + u < nw, m4[u], d4[u], true);
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            const float mn = fmaxf(m[r], fmaxf(m4[0][r], m4[1][r]));
            if (mn == -INFINITY) continue;
            float acc = d[r] * ptx::ex2(m[r] - mn);  // ex2(-inf) = 0 while nothing was seen yet
#pragma unroll
            for (int u = 0; u < kFold; ++u) acc = fmaf(d4[u][r], ptx::ex2(m4[u][r] - mn), acc);
            m[r] = mn;
            d[r] = acc;
        }
    }
    // the team's (m, d) of each row: m = max_w m_w, d = sum_w 2^{m_w - m} d_w
    float mneg[4], inv_d[4];
    if constexpr (TW > 1) {
        part_m[warp][lane] = make_float4(m[0], m[1], m[2], m[3]);
        part_d[warp][lane] = make_float4(d[0], d[1], d[2], d[3]);
        __syncthreads();  // the whole CTA is one class: uniform
        float M[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY}, D[4] = {0.f, 0.f, 0.f, 0.f};
        const int w0 = team * TW;
#pragma unroll
        for (int w = 0; w < TW; ++w) {
            const float4 pm = part_m[w0 + w][lane];
            M[0] = fmaxf(M[0], pm.x); M[1] = fmaxf(M[1], pm.y); M[2] = fmaxf(M[2], pm.z); M[3] = fmaxf(M[3], pm.w);
        }
#pragma unroll
        for (int r = 0; r < 4; ++r) mneg[r] = M[r] == -INFINITY ? 0.f : -M[r];
#pragma unroll
        for (int w = 0; w < TW; ++w) {
            const float4 pm = part_m[w0 + w][lane], pd = part_d[w0 + w][lane];
            D[0] = fmaf(pd.x, ptx::ex2(pm.x + mneg[0]), D[0]);
            D[1] = fmaf(pd.y, ptx::ex2(pm.y + mneg[1]), D[1]);
            D[2] = fmaf(pd.z, ptx::ex2(pm.z + mneg[2]), D[2]);
            D[3] = fmaf(pd.w, ptx::ex2(pm.w + mneg[3]), D[3]);
        }
#pragma unroll
        for (int r = 0; r < 4; ++r) inv_d[r] = D[r] > 0.f ? 1.f / D[r] : 0.f;
    } else {
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            mneg[r] = m[r] == -INFINITY ? 0.f : -m[r];  // all-masked row: every term is 0
            inv_d[r] = d[r] > 0.f ? 1.f / d[r] : 0.f;
        }
    }
    // r'_k = e_k * 2^{m_w - m} / d for the kept tiles (e_k = 0 wherever m'_k = -inf, and a warp that
    // saw no valid tile has m_w = -inf: factor 0, never inf * 0)
    float fac[4];
#pragma unroll
    for (int r = 0; r < 4; ++r) fac[r] = mw[r] == -INFINITY ? 0.f : ptx::ex2(mw[r] + mneg[r]) * inv_d[r];
#pragma unroll
    for (int u = 0; u < KR; ++u)
        if (u < nw) {
            float s4[4];
#pragma unroll
            for (int r = 0; r < 4; ++r) s4[r] = mk[u][r] * fac[r];
            ir_store(rp, u * TW, s4);
        }
    for (int tb = KR; tb < nw; tb += kFold) {  // the folded tiles: m' re-read, r'_k = 2^{m'_k - m} / d
        float m4[kFold][4], d4[kFold][4];
#pragma unroll
        for (int u = 0; u < kFold; ++u) ir_load(mp, dp, ti, hbit, (tb + u) * TW, tb + u < nw, m4[u], d4[u], false);
#pragma unroll
        for (int u = 0; u < kFold; ++u)
            if (tb + u < nw) {
                float s4[4];
#pragma unroll
                for (int r = 0; r < 4; ++r) s4[r] = ptx::ex2(m4[u][r] + mneg[r]) * inv_d[r];
                ir_store(rp, (tb + u) * TW, s4);
            }
    }
}

template <int KR>
__global__ void __launch_bounds__(kW * 32, SR_IR_MIN_CTAS) ir_kernel(const Params p)
{
    __shared__ float4 part_m[kW][32], part_d[kW][32];
    ptx::griddep_launch_dependents();  // PDL: GEMM2's prologue may start now ...
    ptx::griddep_wait();               // ... and GEMM1's m', d' must be complete before we read them
    // this CTA's class c (team size 8 >> c, 1 << c row-blocks per CTA) and its first row-block
    int b = blockIdx.x, first = 0, c = 0;
    for (; c < 4; ++c) {
        const int nc = p.sc.n_ir_class[c], ncta = (nc + (1 << c) - 1) >> c;
        if (b < ncta) break;
        b -= ncta;
        first += nc;
    }
    if (c == 4) return;  // (not reached: the grid covers the classes exactly)
    const int team = (threadIdx.x / 32) >> (3 - c);
    const int idx = first + (b << c) + team;
    const bool live = idx < first + p.sc.n_ir_class[c];
    switch (c) {
        case 0: ir_team<8, KR>(p, idx, live, part_m, part_d); break;
        case 1: ir_team<4, KR>(p, idx, live, part_m, part_d); break;
        case 2: ir_team<2, KR>(p, idx, live, part_m, part_d); break;
        default: ir_team<1, KR>(p, idx, live, part_m, part_d); break;
    }
}

cudaError_t launch_ir(const Params& p, cudaStream_t st, int64_t* nlaunch)
{
    int64_t blocks = 0;  // per class c (team size 8 >> c): ceil(rows / (8 / team size)) CTAs
    for (int c = 0; c < 4; ++c) blocks += (p.sc.n_ir_class[c] + (1 << c) - 1) >> c;
    if (blocks == 0) return cudaSuccess;
    // the classes were cut for ir_warp_tiles tiles per warp on the host (make_blob)
    if (p.sc.ir_warp_tiles == kIrWarpTilesWide)
        return launch_pdl(ir_kernel<kIrWarpTilesWide>, dim3((unsigned)blocks), dim3(kW * 32), 0, st, nlaunch, p);
    return launch_pdl(ir_kernel<kIrWarpTiles>, dim3((unsigned)blocks), dim3(kW * 32), 0, st, nlaunch, p);
}

// ---------------------------------------------------------------- SR_SPLIT_KV combine
// O of a split row-block = the sum of its chunks' partial outputs.  Every chunk already applied the
// row's global Global-Scaling factor r'_k = e^{m'_k - m} / d of its own tiles, so the
// partial contexts add with no rescaling; they are summed in chunk order (deterministic).  One thread
// per 4 output columns of a row.
template <int D>
__global__ void __launch_bounds__(256) combine_kernel(const Params p)
{
    ptx::griddep_launch_dependents();
    ptx::griddep_wait();  // GEMM2's partial rows must be complete
    constexpr int PER = kRowBlock * D / 4;  // float4 per row-block
    const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int j = (int)(idx / PER);
    if (j >= p.sc.n_comb) return;
    const int e = (int)(idx % PER), r = e / (D / 4), c4 = e % (D / 4);
    const int4 cb = __ldcg(p.sc.comb + j);  // {row-block item, first slot, chunks, 0}
    const int g = cb.x / p.sc.n_rb, rb = cb.x % p.sc.n_rb;
    if (rb * kRowBlock + r >= p.S) return;  // a row beyond the head (S % 128 == 64)
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int c = 0; c < cb.z; ++c) {
        const float4 v = __ldcg(reinterpret_cast<const float4*>(p.partial + ((int64_t)(cb.y + c) * kRowBlock + r) * D) + c4);
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    const int64_t orow = (int64_t)g * p.S + rb * kRowBlock + r;
    if (p.out_dtype == DT_F32) {
        reinterpret_cast<float4*>((float*)p.out + orow * D)[c4] = acc;
    } else {
        const bool bf = p.out_dtype == DT_BF16;
        const uint2 w = make_uint2(bf ? ptx::pack_bf16(acc.x, acc.y) : ptx::pack_f16(acc.x, acc.y),
                                   bf ? ptx::pack_bf16(acc.z, acc.w) : ptx::pack_f16(acc.z, acc.w));
        reinterpret_cast<uint2*>((uint16_t*)p.out + orow * D)[c4] = w;
    }
}

cudaError_t launch_combine(const Params& p, cudaStream_t st, int64_t* nlaunch)
{
    if (p.sc.n_comb == 0) return cudaSuccess;
    const int64_t n = (int64_t)p.sc.n_comb * kRowBlock * p.D / 4;
    const dim3 grid((unsigned)((n + 255) / 256));
    return p.D == 64 ? launch_pdl(combine_kernel<64>, grid, dim3(256), 0, st, nlaunch, p)
                     : launch_pdl(combine_kernel<128>, grid, dim3(256), 0, st, nlaunch, p);
}

}  // namespace sr
