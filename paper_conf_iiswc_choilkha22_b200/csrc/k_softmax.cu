// k_softmax.cu -- the unfused baseline's softmax kernel (a row vector per thread
// block held in on-chip memory; the attention matrix is read once and written once).  Part of the
// in-repo traffic baseline only; the recomposed path never runs it.
//
// row_softmax (rows longer than the register-resident kernel below takes, or SR_SOFTMAX_SMEM=1):
// One CTA per (row-block, slice of R rows): every score tile of the row-block holds the slice's R
// rows of each 64-key chunk as R x 128 contiguous bytes (SWIZZLE_128B tile layout), so the CTA pulls
// the slice's whole score rows into shared memory with one bulk copy per chunk (all in flight at
// once), computes the safe softmax of Eq. (1) row by row in place (one warp per row: max, sum of
// exponentials, normalised write), and bulk-stores P back.  R = 32 down to 2, chosen on the host so
// the slice takes <= 48 KB (several CTAs per SM then overlap one CTA's loads with another's
// arithmetic and stores): sized for the longest rows when that leaves R >= 8, else for the mean
// row, and the few longer rows (global tokens) go through shared memory in groups, twice (online
// max and sum, then the normalised write).  A memory-bound kernel meant to run at HBM bandwidth: a fair
// baseline for the fused path's traffic savings.
#include "tc_common.cuh"

namespace sr {

using namespace ptx;

constexpr int kSmBudget = 48 * 1024, kSmBudgetMax = 160 * 1024;

template <int T>
__global__ void __launch_bounds__(256) row_softmax(const Params p, int R, int cap)  // min(R, 8) warps
{
    extern __shared__ __align__(128) uint8_t rows[];  // [chunk][R rows][128 B]
    __shared__ uint64_t bar;
    __shared__ int n_chunks;
    constexpr int XB = kRowBlock * T * 2;
    const DevSched& sc = p.sc;
    const int nsl = kRowBlock / R;
    const int item = blockIdx.x / nsl;  // g * n_rb + rb
    const int r0 = (blockIdx.x % nsl) * R;
    const int g = item / sc.n_rb, rb = item % sc.n_rb;
    const int myhalf = r0 / kHalf;  // R <= 64: the slice lies in one 64-row half
    const int32_t* tp = sc.tp + (size_t)lh_of(sc, g, p.H) * (sc.n_rb + 1);
    griddep_launch_dependents();
    griddep_wait();
    const int t0 = __ldcg(tp + rb), t1 = __ldcg(tp + rb + 1);
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - __ldcg(tp);
    const uint32_t slice = (uint32_t)R * 128;
    // bulk copies of the slice's chunks k0 .. k1-1 (in row order) between HBM and shared memory
    auto copy_chunks = [&](int k0, int k1, bool load) {
        int k = 0;
        for (int t = t0; t < t1 && k < k1; ++t) {
            if (!((tinfo_half(__ldcg(sc.tinfo + t)) >> myhalf) & 1)) continue;
            const int64_t off = (slot0 + t) * (int64_t)XB + r0 * 128;
            for (int ch = 0; ch < T / 64; ++ch, ++k) {
                if (k < k0 || k >= k1) continue;
                uint8_t* sm = rows + (k - k0) * slice;
                if (load) bulk_load(sm, (const uint8_t*)p.xprime + off + ch * (kRowBlock * 128), slice, &bar);
                else bulk_store((uint8_t*)p.pbuf + off + ch * (kRowBlock * 128), sm, slice);
            }
        }
    };
    if (threadIdx.x == 0) {
        int n = 0;
        for (int t = t0; t < t1; ++t) n += ((tinfo_half(__ldcg(sc.tinfo + t)) >> myhalf) & 1) ? T / 64 : 0;
        n_chunks = n;
        mbar_init(&bar, 1);
        fence_mbar_init();
        if (n) {
            mbar_arrive_expect_tx(&bar, min(n, cap) * slice);
            copy_chunks(0, min(n, cap), true);
        }
    }
    __syncthreads();
    const int nck = n_chunks;
    if (nck == 0) return;
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const float l2e = 1.4426950408889634f;
    const bool bf = p.in_dtype == DT_BF16;
    const int nwarps = blockDim.x / 32;
    const int ngrp = (nck + cap - 1) / cap;  // > 1: rows longer than the slice capacity
    if (ngrp == 1) {  // the whole row slice is on chip: max, then e = e^{x - m} (kept, fp16) and its
                      // sum, then P = e / sum -- one exponential per element
        mbar_wait(&bar, 0);
        for (int rr = warp; rr < R; rr += nwarps) {
            const uint32_t base = smem_u32(rows) + rr * 128 + lane * 4;  // lane: 2 keys of every chunk
            float m = -INFINITY;
            for (int k = 0; k < nck; ++k) {
                const float2 f = unpack_f16(lds_u32(base + k * slice));
                m = fmaxf(m, fmaxf(f.x, f.y));
            }
            for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
            const float neg = m == -INFINITY ? 0.f : -m * l2e;
            float s = 0.f;
            for (int k = 0; k < nck; ++k) {
                const float2 f = unpack_f16(lds_u32(base + k * slice));
                const float e0 = ex2(fmaf(f.x, l2e, neg)), e1 = ex2(fmaf(f.y, l2e, neg));
                s += e0 + e1;
                sts_u32(base + k * slice, pack_f16(e0, e1));
            }
            for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
            const float inv = s > 0.f ? 1.f / s : 0.f;
            for (int k = 0; k < nck; ++k) {
                const float2 e = unpack_f16(lds_u32(base + k * slice));
                sts_u32(base + k * slice, bf ? pack_bf16(e.x * inv, e.y * inv) : pack_f16(e.x * inv, e.y * inv));
            }
        }
        fence_proxy_async_smem();
        __syncthreads();
        if (threadIdx.x == 0) {
            copy_chunks(0, nck, false);
            bulk_commit();
            bulk_wait_read0();
        }
        return;
    }
    uint32_t ph = 0;
    // rows longer than the slice: pass 1 over groups of `cap` chunks, per-lane online max and sum
    float mx[4], sm_[4];  // rows warp + 8j of this warp (R <= 32, nwarps = min(R, 8))
#pragma unroll
    for (int j = 0; j < 4; ++j) { mx[j] = -INFINITY; sm_[j] = 0.f; }
    for (int gi = 0; gi < ngrp; ++gi) {
        const int nk = min(cap, nck - gi * cap);
        if (gi > 0) {
            __syncthreads();  // everyone is done with the previous group
            if (threadIdx.x == 0) {
                mbar_arrive_expect_tx(&bar, nk * slice);
                copy_chunks(gi * cap, gi * cap + nk, true);
            }
        }
        mbar_wait(&bar, ph);
        ph ^= 1;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int rr = warp + j * nwarps;
            if (rr >= R) break;
            const uint32_t base = smem_u32(rows) + rr * 128 + lane * 4;  // lane: 2 keys of every chunk
            float m = mx[j];
            for (int k = 0; k < nk; ++k) {
                const float2 f = unpack_f16(lds_u32(base + k * slice));
                m = fmaxf(m, fmaxf(f.x, f.y));
            }
            const float neg = m == -INFINITY ? 0.f : -m * l2e;
            float s = mx[j] == -INFINITY ? 0.f : sm_[j] * ex2(fmaf(mx[j], l2e, neg));
            for (int k = 0; k < nk; ++k) {
                const float2 f = unpack_f16(lds_u32(base + k * slice));
                s += ex2(fmaf(f.x, l2e, neg)) + ex2(fmaf(f.y, l2e, neg));
            }
            mx[j] = m;
            sm_[j] = s;
        }
    }
    // warp reductions of the row statistics
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        float m = mx[j];
        for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
        float s = mx[j] == -INFINITY ? 0.f : sm_[j] * ex2((mx[j] - m) * l2e);
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        mx[j] = m == -INFINITY ? 0.f : -m * l2e;  // now: the exponent offset
        sm_[j] = s > 0.f ? 1.f / s : 0.f;          // now: 1 / row sum
    }
    // pass 2: P = e^{x - m} / d, in place, then out with bulk stores (re-loading groups if needed)
    for (int gi = 0; gi < ngrp; ++gi) {
        const int nk = min(cap, nck - gi * cap);
        if (ngrp > 1) {
            __syncthreads();
            if (threadIdx.x == 0) {
                if (gi > 0) bulk_wait_read0();  // the previous group's stores have left shared memory
                mbar_arrive_expect_tx(&bar, nk * slice);
                copy_chunks(gi * cap, gi * cap + nk, true);
            }
            __syncthreads();
            mbar_wait(&bar, ph);
            ph ^= 1;
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int rr = warp + j * nwarps;
            if (rr >= R) break;
            const uint32_t base = smem_u32(rows) + rr * 128 + lane * 4;
            for (int k = 0; k < nk; ++k) {
                const float2 f = unpack_f16(lds_u32(base + k * slice));
                const float y0 = ex2(fmaf(f.x, l2e, mx[j])) * sm_[j], y1 = ex2(fmaf(f.y, l2e, mx[j])) * sm_[j];
                sts_u32(base + k * slice, bf ? pack_bf16(y0, y1) : pack_f16(y0, y1));
            }
        }
        fence_proxy_async_smem();
        __syncthreads();
        if (threadIdx.x == 0) {
            copy_chunks(gi * cap, gi * cap + nk, false);
            bulk_commit();
        }
    }
    if (threadIdx.x == 0) bulk_wait_read0();
}

// ---------------------------------------------------------------- register-resident row softmax
// The default baseline softmax for rows of up to 4 * kNiMax 64-key chunks (4096 keys): one CTA per
// (row-block, 64-row half) -- the rows of a half share one list of stored tiles -- and one warp per
// row at a time.  A warp-wide 16-B load covers 4 chunks x 128 B of its row (lane l: chunk l/8,
// 16-B piece l%8 of the SWIZZLE_128B row), so a row of up to 4*NI chunks sits in 4*NI registers per
// lane: the scores are read once and P written once straight from registers, every
// load of a row in flight at once.  Arithmetic in packed fp16 (max, exponent argument, ex2.f16x2,
// normalisation; the row sum accumulates in fp32): ~3 instructions per element.  Scores are the
// fp16 values GEMM1 stored; masked ones are -inf; a row with no kept key writes zeros.
constexpr int kNiMax = 16;

__device__ __forceinline__ __half2 u2h(uint32_t w) { return *reinterpret_cast<__half2*>(&w); }
__device__ __forceinline__ uint32_t h2u(__half2 h) { return *reinterpret_cast<uint32_t*>(&h); }
__device__ __forceinline__ __half2 ex2_h2(__half2 t)  // one MUFU op for two fp16 results
{
    uint32_t y;
    asm("ex2.approx.f16x2 %0, %1;" : "=r"(y) : "r"(h2u(t)));
    return u2h(y);
}

// LONG: the launch for the halves listed in sc.sm_long (rows of more than kSmShortChunks chunks): each
// CTA takes kLongRows of a listed half's 64 rows, one row per warp, so the few long rows of a layer
// (global tokens) spread over many SMs instead of 8 warps walking 64 rows in turn.
constexpr int kLongRows = 8;

template <int T, int NI, bool BF, bool LONG = false>
__global__ void __launch_bounds__(256) row_softmax_reg(const Params p, int lo, int hi, int rsplit)  // halves with lo < chunks <= hi
{
    __shared__ int64_t slot_list[1024];  // stored tiles of this half, as slot ids
    __shared__ int n_tiles;
    constexpr int XB = kRowBlock * T * 2, CPT = T / 64;
    const DevSched& sc = p.sc;
    // a half's 64 rows over rsplit CTAs (LONG: kHalf / kLongRows): more, smaller CTAs shorten the
    // grid's last partial wave
    const int rs = LONG ? kHalf / kLongRows : rsplit;
    const int hsel = LONG ? __ldcg(sc.sm_long + blockIdx.x / rs) : (int)(blockIdx.x / rs);
    const int item = hsel >> 1, half = hsel & 1;  // item = g * n_rb + rb
    const int row_lo = (int)(blockIdx.x % rs) * (kHalf / rs);
    const int row_hi = row_lo + kHalf / rs;
    const int g = item / sc.n_rb, rb = item % sc.n_rb;
    const int32_t* tp = sc.tp + (size_t)lh_of(sc, g, p.H) * (sc.n_rb + 1);
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    griddep_launch_dependents();
    griddep_wait();
    const int t0 = __ldcg(tp + rb), t1 = __ldcg(tp + rb + 1);
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - __ldcg(tp);
    if (warp == 0) {  // compact the tiles whose `half` is valid (ballot + prefix, 32 at a time)
        int n = 0;
        for (int tb = t0; tb < t1; tb += 32) {
            const int t = tb + lane;
            const bool v = t < t1 && ((tinfo_half(__ldcg(sc.tinfo + t)) >> half) & 1);
            const unsigned m = __ballot_sync(0xffffffffu, v);
            if (v) slot_list[n + __popc(m & ((1u << lane) - 1))] = slot0 + t;
            n += __popc(m);
        }
        if (lane == 0) n_tiles = n;
    }
    __syncthreads();
    const int nch = n_tiles * CPT;  // 64-key chunks of each row of this half
    if (!LONG && (nch <= lo || nch > hi)) return;  // another launch's length class (or nothing stored)
    const int sub = lane >> 3;  // chunk within a group of 4
    const int ni = (nch + 3) / 4;  // 16-B words per lane actually used by this half's rows (warp-uniform)
    const __half2 l2e = __float2half2_rn(1.4426950408889634f);
    // NR rows of the warp in flight at once (short rows: more of them, so a warp keeps ~8 loads out)
    constexpr int NR = NI >= 8 ? 1 : 8 / NI;
    for (int rr0 = row_lo + warp * NR; rr0 < row_hi; rr0 += 8 * NR) {
        uint4 x[NR][NI];
        int64_t base[NR];
#pragma unroll
        for (int q = 0; q < NR; ++q) {
            const int r = half * kHalf + rr0 + q;
            base[q] = (int64_t)r * 128 + (int64_t)((((lane & 7) ^ (r & 7))) << 4);
#pragma unroll
            for (int i = 0; i < NI; ++i) {  // every load of the NR rows in flight at once
                const int k = 4 * i + sub;
                x[q][i] = make_uint4(0xFC00FC00u, 0xFC00FC00u, 0xFC00FC00u, 0xFC00FC00u);  // -inf (fp16)
                if (k < nch)
                    x[q][i] = __ldcg(reinterpret_cast<const uint4*>((const uint8_t*)p.xprime + slot_list[k / CPT] * (int64_t)XB +
                                                                   (k % CPT) * (kRowBlock * 128) + base[q]));
            }
        }
#pragma unroll
        for (int q = 0; q < NR; ++q) {
            __half2 m2 = u2h(0xFC00FC00u);
#pragma unroll
            for (int i = 0; i < NI; ++i)
                if (i < ni)  // warp-uniform: only the words this half's rows use
                    m2 = __hmax2(__hmax2(m2, __hmax2(u2h(x[q][i].x), u2h(x[q][i].y))),
                                 __hmax2(u2h(x[q][i].z), u2h(x[q][i].w)));
            float m = fmaxf(__low2float(m2), __high2float(m2));
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
            // exponent argument (x - m) * log2(e) in fp16: x and m are fp16 values, so x - m is exact
            // up to one rounding; 2^t on MUFU (fully masked row: every t is -inf -> 0)
            const __half2 nm = __float2half2_rn(m == -INFINITY ? 0.f : -m);
            float s0 = 0.f, s1 = 0.f;
#pragma unroll
            for (int i = 0; i < NI; ++i) {
                if (i >= ni) continue;
                __half2 e[4] = {u2h(x[q][i].x), u2h(x[q][i].y), u2h(x[q][i].z), u2h(x[q][i].w)};
#pragma unroll
                for (int u = 0; u < 4; ++u) e[u] = ex2_h2(__hmul2(__hadd2(e[u], nm), l2e));
                const float2 f = __half22float2(__hadd2(__hadd2(e[0], e[1]), __hadd2(e[2], e[3])));
                s0 += f.x;
                s1 += f.y;
                x[q][i] = make_uint4(h2u(e[0]), h2u(e[1]), h2u(e[2]), h2u(e[3]));
            }
            float sum = s0 + s1;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
            const float inv = sum > 0.f ? 1.f / sum : 0.f;
            const __half2 inv2 = __float2half2_rn(inv);
#pragma unroll
            for (int i = 0; i < NI; ++i) {
                const int k = 4 * i + sub;
                if (i >= ni || k >= nch) continue;
                uint32_t w[4] = {x[q][i].x, x[q][i].y, x[q][i].z, x[q][i].w};
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    if constexpr (BF) {
                        const float2 f = __half22float2(u2h(w[u]));
                        w[u] = pack_bf16(f.x * inv, f.y * inv);
                    } else {
                        w[u] = h2u(__hmul2(u2h(w[u]), inv2));
                    }
                }
                stg128((uint8_t*)p.pbuf + slot_list[k / CPT] * (int64_t)XB + (k % CPT) * (kRowBlock * 128) + base[q],
                       w[0], w[1], w[2], w[3]);
            }
        }
    }
}

// rows per CTA and slice capacity in chunks: the largest power of two R <= 32 whose slice fits 48 KB,
// for the longest rows if that gives R >= 8, else for the mean row (2 rows in up to 160 KB at worst)
static void softmax_shape(const DevSched& sc, int T, int* R_, int* cap_)
{
    const size_t nmax = (size_t)std::max(1, sc.max_rb_tiles * (T / 64));
    const size_t nmean = (size_t)std::max(1, sc.mean_rb_tiles * (T / 64));
    int R = 0;
    for (int r = 32; r >= 8 && !R; r /= 2)
        if (nmax * r * 128 <= (size_t)kSmBudget) R = r;
    if (R) { *R_ = R; *cap_ = (int)nmax; return; }
    for (int r = 32; r >= 2 && !R; r /= 2)
        if (nmean * r * 128 <= (size_t)kSmBudget) R = r;
    if (R) { *R_ = R; *cap_ = kSmBudget / (R * 128); return; }
    *R_ = 2;
    *cap_ = (int)std::min(nmax, (size_t)kSmBudgetMax / 256);
}

template <int T>
cudaError_t launch_softmax_t(const Params& p, cudaStream_t st, int64_t* nl)
{
    int R, cap;
    softmax_shape(p.sc, T, &R, &cap);
    const size_t sm = (size_t)cap * R * 128;
    cudaError_t e = cudaFuncSetAttribute(row_softmax<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    const int64_t blocks = (int64_t)p.B * p.H * p.sc.n_rb * (kRowBlock / R);
    return launch_pdl(row_softmax<T>, dim3((unsigned)blocks), dim3(32 * std::min(R, 8)), sm, st, nl, p, R, cap);
}

template <int T, bool BF>
cudaError_t launch_softmax_reg(const Params& p, cudaStream_t st, int64_t* nl, int ni, int lo, int hi)
{
    static const int env_rs = [] { const char* e = getenv("SR_SOFTMAX_RSPLIT"); return e ? atoi(e) : 0; }();
    // rows of 17-32 chunks (one row per warp at a time): two CTAs per half (measured, back to back:
    // C3 107.2 -> 101.9 us); shorter rows keep one (C2, C4-C6 within noise or slower split)
    int rs = env_rs == 1 || env_rs == 2 || env_rs == 4 || env_rs == 8 ? env_rs : (ni == 8 ? 2 : 1);
    // a CTA's rows must be whole iterations of its 8 warps x NR rows (NR = 8 / NI rows below NI = 8)
    rs = std::min(rs, ni >= 8 ? 8 : ni);
    const dim3 grid((unsigned)((int64_t)p.B * p.H * p.sc.n_rb * 2 * rs));
    switch (ni) {
    case 2: return launch_pdl(row_softmax_reg<T, 2, BF>, grid, dim3(256), 0, st, nl, p, lo, hi, rs);
    case 4: return launch_pdl(row_softmax_reg<T, 4, BF>, grid, dim3(256), 0, st, nl, p, lo, hi, rs);
    case 8: return launch_pdl(row_softmax_reg<T, 8, BF>, grid, dim3(256), 0, st, nl, p, lo, hi, rs);
    default: return launch_pdl(row_softmax_reg<T, 16, BF>, grid, dim3(256), 0, st, nl, p, lo, hi, rs);
    }
}

template <int T, bool BF>
cudaError_t launch_softmax_classes(const Params& p, cudaStream_t st, int64_t* nl, int max_ch)
{
    // rows of <= kSmShortChunks chunks with a short-row instantiation (several rows in flight per
    // warp); the halves with longer rows (global rows of BigBird / Longformer) with a second launch
    // over their list, kLongRows rows per CTA (C4 softmax 130 -> 99 us)
    int ni = 2;
    while (4 * ni < max_ch) ni *= 2;
    if (ni <= 8) return launch_softmax_reg<T, BF>(p, st, nl, ni, 0, INT32_MAX);
    cudaError_t e = launch_softmax_reg<T, BF>(p, st, nl, 4, 0, kSmShortChunks);
    if (e != cudaSuccess || p.sc.n_sm_long == 0) return e;
    const dim3 grid((unsigned)((int64_t)p.sc.n_sm_long * (kHalf / kLongRows)));
    return ni == 16 ? launch_pdl(row_softmax_reg<T, 16, BF, true>, grid, dim3(256), 0, st, nl, p, 0, 0, 0)
                    : launch_pdl(row_softmax_reg<T, 8, BF, true>, grid, dim3(256), 0, st, nl, p, 0, 0, 0);
}

cudaError_t launch_softmax(const Params& p, cudaStream_t st, int64_t* nl)
{
    // rows of up to 4 * kNiMax chunks (4096 keys): the register-resident kernel; longer rows stream
    // through shared memory (row_softmax).  SR_SOFTMAX_SMEM=1 forces the latter (experiments).
    const int max_ch = p.sc.max_rb_tiles * (p.T / 64);
    static const bool force_smem = getenv("SR_SOFTMAX_SMEM") != nullptr;
    if (!force_smem && max_ch <= 4 * kNiMax && p.sc.max_rb_tiles <= 1024) {
        const bool bf = p.in_dtype == DT_BF16;
        if (p.T == 64) return bf ? launch_softmax_classes<64, true>(p, st, nl, max_ch) : launch_softmax_classes<64, false>(p, st, nl, max_ch);
        return bf ? launch_softmax_classes<128, true>(p, st, nl, max_ch) : launch_softmax_classes<128, false>(p, st, nl, max_ch);
    }
    return p.T == 64 ? launch_softmax_t<64>(p, st, nl) : launch_softmax_t<128>(p, st, nl);
}

}  // namespace sr
