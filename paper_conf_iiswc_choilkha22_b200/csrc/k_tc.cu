// k_tc.cu -- tcgen05 / TMEM / TMA kernels of the recomposed chain and of the unfused baseline.
//
//   tc_gemm1<D, T, LS=true>   GEMM1 + scale + mask + Local Softmax
//   tc_gemm1<D, T, LS=false>  unfused baseline GEMM1: scale + mask, writes the score tile S (L171)
//   tc_gemm2<D, T, GS=true>   Global Scaling fused into GEMM2's prologue (L151, L165) + P.V
//   tc_gemm2<D, T, GS=false>  unfused baseline GEMM2: P.V on the softmax output P
//   row_softmax               unfused baseline softmax, one warp per row (L102)
//
// Both GEMMs are persistent, warp-specialised kernels (one CTA per SM, static longest-first item
// order):  warp 0 = TMA producer, warp 1 = tcgen05.mma issuer (one thread), warp 2 = TMEM
// allocator, warps 4.. = epilogue / transform warpgroups.  Accumulators live in TMEM; smem stages,
// TMEM buffers and the epilogue are chained with mbarriers (full/empty pairs).  Tiles of the
// attention matrix (X', S, P) are stored in the canonical SWIZZLE_128B K-major layout
// [T/64][128 rows][64 cols] so a whole tile moves HBM <-> smem with 1-D bulk copies and GEMM2 can
// feed it to the tensor core without re-layout.
#include <cuda.h>

#include <mutex>

#include "ptx.cuh"
#include "sr_internal.h"

namespace sr {

using namespace ptx;

// ============================================================================ common helpers

struct ItemInfo {
    int g, rb, t0, t1;
    int64_t slot0;  // slot id of tile t is slot0 + t
};

__device__ __forceinline__ ItemInfo decode_item(const Params& p, int it)
{
    const DevSched& sc = p.sc;
    const int item = __ldg(sc.items + it);
    ItemInfo r;
    r.g = item / sc.n_rb;
    r.rb = item % sc.n_rb;
    const int lh = lh_of(sc, r.g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    r.t0 = __ldg(tp + r.rb);
    r.t1 = __ldg(tp + r.rb + 1);
    r.slot0 = (int64_t)r.g * sc.slots_per_head - __ldg(tp);
    return r;
}

// byte offset of 16-B chunk `c` (logical, 0 .. T/8-1) of row r inside a SW128 K-major tile
__device__ __forceinline__ uint32_t tile_chunk_off(int r, int c)
{
    return (uint32_t)((c >> 3) * (kRowBlock * 128) + r * 128 + (((c & 7) ^ (r & 7)) << 4));
}

constexpr int kSmemMax = 232448;  // 227 KB opt-in dynamic shared memory per CTA on sm_100

// ============================================================================ GEMM1

template <int D, int T>
struct G1 {
    static constexpr int QB = kRowBlock * D * 2;  // Q tile bytes
    static constexpr int KB = T * D * 2;          // K tile bytes
    static constexpr int XB = kRowBlock * T * 2;  // X'/S tile bytes (one staging buffer per WG)
    static constexpr int NQ = 2;
    static constexpr int NACC = 512 / T;  // TMEM accumulator buffers (4 for T=128, 8 for T=64)
    static constexpr int NK_ = (kSmemMax - 2048 - NQ * QB - 2 * XB) / KB;
    static constexpr int NK = NK_ > 4 ? 4 : NK_;
    static_assert(NK >= 2, "smem budget");
    static constexpr int OFF_Q = 0;
    static constexpr int OFF_K = OFF_Q + NQ * QB;
    static constexpr int OFF_X = OFF_K + NK * KB;
    static constexpr int OFF_BAR = OFF_X + 2 * XB;
    static constexpr int NBAR = 2 * NQ + 2 * NK + 2 * NACC;
    static constexpr int SMEM_ = OFF_BAR + NBAR * 8 + 16 + 1024;  // + tmem ptr + alignment slack
    static constexpr int SMEM = SMEM_ > 118 * 1024 ? SMEM_ : 118 * 1024;  // 1 CTA/SM (512 TMEM cols)
    static constexpr int THREADS = 384;
};

template <int D, int T, bool LS>
__global__ void __launch_bounds__(384, 1)
    tc_gemm1(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK, const Params p)
{
    using C = G1<D, T>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint64_t* bars = (uint64_t*)(smem + C::OFF_BAR);
    uint64_t* q_full = bars;
    uint64_t* q_empty = q_full + C::NQ;
    uint64_t* k_full = q_empty + C::NQ;
    uint64_t* k_empty = k_full + C::NK;
    uint64_t* acc_full = k_empty + C::NK;
    uint64_t* acc_empty = acc_full + C::NACC;
    uint32_t* tmem_ptr = (uint32_t*)(acc_empty + C::NACC);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (threadIdx.x == 0) {
        for (int i = 0; i < C::NQ; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
        for (int i = 0; i < C::NK; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
        for (int i = 0; i < C::NACC; ++i) { mbar_init(&acc_full[i], 1); mbar_init(&acc_empty[i], 4); }
        fence_mbar_init();
    }
    if (warp == 0 && lane == 0) { prefetch_tmap(&tmQ); prefetch_tmap(&tmK); }
    if (warp == 2) tmem_alloc(tmem_ptr, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_ptr;
    const int n_items = p.sc.n_items;
    // 168 regs/thread at launch; warpgroup 0 (producer, MMA, allocator) hands registers to the
    // two epilogue warpgroups, which hold a whole 128 x T fp32 row block each
    if (warp < 4) {
    reg_dealloc<56>();
    if (warp == 0) {
        // ------------------------------------------------------------------ TMA producer
        if (lane == 0) {
            int qi = 0, ks = 0;
            uint32_t qph = 0, kph = 0;
            for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
                const ItemInfo I = decode_item(p, it);
                if (I.t0 == I.t1) continue;
                const int row0 = I.g * p.S + I.rb * kRowBlock;
                mbar_wait(&q_empty[qi], qph ^ 1);
                mbar_arrive_expect_tx(&q_full[qi], C::QB);
                for (int h = 0; h < D / 64; ++h)
                    tma_load_2d(smem + C::OFF_Q + qi * C::QB + h * (kRowBlock * 128), &tmQ, h * 64, row0, &q_full[qi]);
                if (++qi == C::NQ) { qi = 0; qph ^= 1; }
                for (int t = I.t0; t < I.t1; ++t) {
                    const int kt = tinfo_kt(__ldg(p.sc.tinfo + t));
                    mbar_wait(&k_empty[ks], kph ^ 1);
                    mbar_arrive_expect_tx(&k_full[ks], C::KB);
                    for (int h = 0; h < D / 64; ++h)
                        tma_load_2d(smem + C::OFF_K + ks * C::KB + h * (T * 128), &tmK, h * 64, I.g * p.S + kt * T,
                                    &k_full[ks]);
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        // ------------------------------------------------------------------ MMA issuer
        if (lane == 0) {
            constexpr uint32_t idesc_f16v = idesc_f16(0, kRowBlock, T, 0, 0);
            constexpr uint32_t idesc_bf16v = idesc_f16(1, kRowBlock, T, 0, 0);
            const uint32_t idesc = p.in_dtype == DT_BF16 ? idesc_bf16v : idesc_f16v;
            int qi = 0, ks = 0, ab = 0;
            uint32_t qph = 0, kph = 0, aph = 0;
            for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
                const ItemInfo I = decode_item(p, it);
                if (I.t0 == I.t1) continue;
                mbar_wait(&q_full[qi], qph);
                tc_fence_after();
                const uint32_t q_addr = smem_u32(smem + C::OFF_Q + qi * C::QB);
                for (int t = I.t0; t < I.t1; ++t) {
                    mbar_wait(&acc_empty[ab], aph ^ 1);
                    mbar_wait(&k_full[ks], kph);
                    tc_fence_after();
                    const uint32_t k_addr = smem_u32(smem + C::OFF_K + ks * C::KB);
                    const uint32_t d_tmem = tmem_base + ab * T;
#pragma unroll
                    for (int kk = 0; kk < D / 16; ++kk) {
                        const uint32_t h = kk / 4, w = kk % 4;
                        const uint64_t ad = smem_desc_sw128(q_addr + h * (kRowBlock * 128) + w * 32, 16, 1024);
                        const uint64_t bd = smem_desc_sw128(k_addr + h * (T * 128) + w * 32, 16, 1024);
                        mma_ss(d_tmem, ad, bd, idesc, kk > 0 ? 1u : 0u);
                    }
                    mma_commit(&k_empty[ks]);
                    mma_commit(&acc_full[ab]);
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                    if (++ab == C::NACC) { ab = 0; aph ^= 1; }
                }
                mma_commit(&q_empty[qi]);
                if (++qi == C::NQ) { qi = 0; qph ^= 1; }
            }
        }
    }
    } else {
        reg_alloc<224>();
        // ------------------------------------------------------------------ epilogue warpgroups
        const int e = (warp - 4) / 4;                 // warpgroup 0 / 1: even / odd tiles
        const int r = (warp % 4) * 32 + lane;         // tile row == TMEM lane
        const int myhalf = r / kHalf;
        uint8_t* stage = smem + C::OFF_X + e * C::XB;
        const uint32_t lane_off = (uint32_t)((warp % 4) * 32) << 16;
        const bool issuer = (threadIdx.x % 128) == 0;
        const float sl2 = p.scale_log2;
        int n = 0;
        for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
            const ItemInfo I = decode_item(p, it);
            const int i = I.rb * kRowBlock + r;
            const int kvl = p.sc.kv_len ? __ldg(p.sc.kv_len + I.g / p.H) : p.S;
            for (int t = I.t0; t < I.t1; ++t, ++n) {
                if ((n & 1) != e) continue;
                const int buf = n % C::NACC;
                const uint32_t ph = (uint32_t)(n / C::NACC) & 1;
                const int w = __ldg(p.sc.tinfo + t);
                const int kt = tinfo_kt(w), hv = tinfo_half(w);
                const bool valid = (hv >> myhalf) & 1;
                const int c0 = kt * T;
                const bool full = c0 + T - 1 < kvl && (!p.causal || c0 + T - 1 <= i) &&
                                  (p.mask_kind != MK_WINDOW || i < p.n_global ||
                                   (i - c0 <= p.win_half && c0 + T - 1 - i <= p.win_half));
                const uint32_t taddr = tmem_base + lane_off + buf * T;
                mbar_wait(&acc_full[buf], ph);
                tc_fence_after();
                // one TMEM read of the whole 128 x T fp32 row block; the accumulator buffer is
                // released to the MMA warp before any math
                uint32_t xr[T];
                if (valid) {
#pragma unroll
                    for (int c = 0; c < T / 32; ++c) tmem_ld32(taddr + c * 32, *reinterpret_cast<uint32_t(*)[32]>(&xr[c * 32]));
                    tmem_wait_ld();
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&acc_empty[buf]);
                // the warpgroup's staging buffer must be free: its previous bulk store has read it
                if (issuer) bulk_wait_read0();
                named_bar_sync(1 + e, 128);
                float mx = -INFINITY, dsum = 0.f;
                if (valid) {
                    if (!full) {  // edge tile: element mask (padding / causal diagonal / band edge)
#pragma unroll
                        for (int u = 0; u < T; ++u)
                            if (!elem_kept(p, kvl, i, c0 + u)) xr[u] = 0xff800000u;  // -inf
                    }
                    float neg = 0.f;
                    if (LS) {
                        float m8[8];
#pragma unroll
                        for (int a = 0; a < 8; ++a) m8[a] = __uint_as_float(xr[a]);
#pragma unroll
                        for (int u = 8; u < T; ++u) m8[u & 7] = fmaxf(m8[u & 7], __uint_as_float(xr[u]));
                        mx = fmaxf(fmaxf(fmaxf(m8[0], m8[1]), fmaxf(m8[2], m8[3])),
                                   fmaxf(fmaxf(m8[4], m8[5]), fmaxf(m8[6], m8[7])));
                        // X' = e^{x - m'} in base 2, log2(e) folded into the scale
                        neg = (mx == -INFINITY) ? 0.f : -mx * sl2;
                    }
                    float s4[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                    for (int q4 = 0; q4 < T / 8; ++q4) {  // 8 scores -> one 16-B chunk of the tile
                        uint32_t w4[4];
#pragma unroll
                        for (int u = 0; u < 4; ++u) {
                            const float x0 = __uint_as_float(xr[q4 * 8 + 2 * u]);
                            const float x1 = __uint_as_float(xr[q4 * 8 + 2 * u + 1]);
                            if (LS) {
                                const float y0 = ex2(fmaf(x0, sl2, neg)), y1 = ex2(fmaf(x1, sl2, neg));
                                s4[u] += y0 + y1;
                                w4[u] = pack_f16(y0, y1);
                            } else {  // unfused baseline: the scaled, masked score
                                w4[u] = pack_f16(x0 * p.scale, x1 * p.scale);
                            }
                        }
                        *reinterpret_cast<uint4*>(stage + tile_chunk_off(r, q4)) = make_uint4(w4[0], w4[1], w4[2], w4[3]);
                    }
                    dsum = (s4[0] + s4[1]) + (s4[2] + s4[3]);
                }
                fence_proxy_async_smem();
                named_bar_sync(1 + e, 128);
                const int64_t slot = I.slot0 + t;
                if (issuer) {
                    uint8_t* dst = (uint8_t*)p.xprime + slot * (int64_t)C::XB;
                    for (int ch = 0; ch < T / 64; ++ch) {
                        const int o = ch * (kRowBlock * 128);
                        if (hv == 3) bulk_store(dst + o, stage + o, kRowBlock * 128);
                        else {
                            const int o2 = o + (hv == 2 ? kHalf * 128 : 0);
                            bulk_store(dst + o2, stage + o2, kHalf * 128);
                        }
                    }
                    bulk_commit();
                }
                if (LS && valid) {
                    p.mprime[slot * kRowBlock + r] = mx * p.scale;  // m' in natural-log units
                    p.dprime[slot * kRowBlock + r] = dsum;
                }
            }
        }
        if (issuer) bulk_wait0();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

// ============================================================================ GEMM2

template <int D, int T>
struct G2 {
    static constexpr int XB = kRowBlock * T * 2;  // X' / P tile
    static constexpr int VB = T * D * 2;          // V tile
    static constexpr int RB = 1024;               // r' of the tile (128 floats), padded to 1 KB
    static constexpr int SB = XB + VB + RB;
    static constexpr int NS_ = (kSmemMax - 2048) / SB;
    static constexpr int NS = NS_ > 4 ? 4 : NS_;
    static_assert(NS >= 2, "smem budget");
    static constexpr int NO = 2;                                  // O accumulators (D cols each)
    static constexpr int NA_ = (512 - NO * D) / (T / 2);          // A operand buffers (T/2 cols)
    static constexpr int NA = NA_ > 8 ? 8 : NA_;
    static_assert(NA >= 2, "tmem budget");
    static constexpr int OFF_S = 0;
    static constexpr int OFF_BAR = NS * SB;
    static constexpr int NBAR = 2 * NS + 2 * NA + 2 * NO;
    static constexpr int SMEM_ = OFF_BAR + NBAR * 8 + 16 + 1024;
    static constexpr int SMEM = SMEM_ > 118 * 1024 ? SMEM_ : 118 * 1024;  // 1 CTA/SM (512 TMEM cols)
    static constexpr int THREADS = 384;
};

template <int D, int T, bool GS>
__global__ void __launch_bounds__(384, 1)
    tc_gemm2(const __grid_constant__ CUtensorMap tmV, const Params p)
{
    using C = G2<D, T>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint64_t* bars = (uint64_t*)(smem + C::OFF_BAR);
    uint64_t* s_full = bars;
    uint64_t* s_empty = s_full + C::NS;
    uint64_t* a_full = s_empty + C::NS;
    uint64_t* a_empty = a_full + C::NA;
    uint64_t* o_full = a_empty + C::NA;
    uint64_t* o_empty = o_full + C::NO;
    uint32_t* tmem_ptr = (uint32_t*)(o_empty + C::NO);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (threadIdx.x == 0) {
        for (int i = 0; i < C::NS; ++i) { mbar_init(&s_full[i], 1); mbar_init(&s_empty[i], 1); }
        for (int i = 0; i < C::NA; ++i) { mbar_init(&a_full[i], 4); mbar_init(&a_empty[i], 1); }
        for (int i = 0; i < C::NO; ++i) { mbar_init(&o_full[i], 1); mbar_init(&o_empty[i], 4); }
        fence_mbar_init();
    }
    if (warp == 0 && lane == 0) prefetch_tmap(&tmV);
    if (warp == 2) tmem_alloc(tmem_ptr, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_ptr;
    const uint32_t tmem_o = tmem_base;              // NO x D columns
    const uint32_t tmem_a = tmem_base + C::NO * D;  // NA x T/2 columns
    const int n_items = p.sc.n_items;
    const void* src = GS ? p.xprime : p.pbuf;

    if (warp == 0) {
        // ------------------------------------------------------------------ producer
        if (lane == 0) {
            int s = 0;
            uint32_t sph = 0;
            for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
                const ItemInfo I = decode_item(p, it);
                for (int t = I.t0; t < I.t1; ++t) {
                    const int w = __ldg(p.sc.tinfo + t);
                    const int kt = tinfo_kt(w), hv = tinfo_half(w);
                    const uint32_t xbytes = (hv == 3 ? 2 : 1) * (T / 64) * (kHalf * 128);
                    mbar_wait(&s_empty[s], sph ^ 1);
                    mbar_arrive_expect_tx(&s_full[s], xbytes + C::VB + (GS ? kRowBlock * 4 : 0));
                    uint8_t* st = smem + C::OFF_S + s * C::SB;
                    const uint8_t* xs = (const uint8_t*)src + (I.slot0 + t) * (int64_t)C::XB;
                    if (hv == 3) bulk_load(st, xs, C::XB, &s_full[s]);
                    else
                        for (int ch = 0; ch < T / 64; ++ch) {
                            const int o = ch * (kRowBlock * 128) + (hv == 2 ? kHalf * 128 : 0);
                            bulk_load(st + o, xs + o, kHalf * 128, &s_full[s]);
                        }
                    for (int h = 0; h < D / 64; ++h)
                        tma_load_2d(st + C::XB + h * (T * 128), &tmV, h * 64, I.g * p.S + kt * T, &s_full[s]);
                    if (GS)  // r' of the tile's 128 rows rides along with the tile (GS operand)
                        bulk_load(st + C::XB + C::VB, p.rprime + (I.slot0 + t) * kRowBlock, kRowBlock * 4, &s_full[s]);
                    if (++s == C::NS) { s = 0; sph ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        // ------------------------------------------------------------------ MMA issuer
        if (lane == 0) {
            constexpr uint32_t idesc_f16v = idesc_f16(0, kRowBlock, D, 0, 1);
            constexpr uint32_t idesc_bf16v = idesc_f16(1, kRowBlock, D, 0, 1);
            const uint32_t idesc = p.in_dtype == DT_BF16 ? idesc_bf16v : idesc_f16v;
            int s = 0, a = 0, o = 0;
            uint32_t sph = 0, aph = 0, oph = 0;
            for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
                const ItemInfo I = decode_item(p, it);
                if (I.t0 == I.t1) continue;
                mbar_wait(&o_empty[o], oph ^ 1);
                tc_fence_after();
                const uint32_t d_tmem = tmem_o + o * D;
                for (int t = I.t0; t < I.t1; ++t) {
                    mbar_wait(&s_full[s], sph);
                    mbar_wait(&a_full[a], aph);
                    tc_fence_after();
                    const uint32_t v_addr = smem_u32(smem + C::OFF_S + s * C::SB + C::XB);
                    const uint32_t a_tm = tmem_a + a * (T / 2);
#pragma unroll
                    for (int kk = 0; kk < T / 16; ++kk) {
                        // B = V tile, MN-major SW128: 16 keys per MMA = 2 KB; 64-wide d blocks at LBO
                        const uint64_t bd = smem_desc_sw128(v_addr + kk * 2048, T * 128, 1024);
                        mma_ts(d_tmem, a_tm + kk * 8, bd, idesc, (t > I.t0 || kk > 0) ? 1u : 0u);
                    }
                    mma_commit(&s_empty[s]);
                    mma_commit(&a_empty[a]);
                    if (++s == C::NS) { s = 0; sph ^= 1; }
                    if (++a == C::NA) { a = 0; aph ^= 1; }
                }
                mma_commit(&o_full[o]);
                if (++o == C::NO) { o = 0; oph ^= 1; }
            }
        }
    } else if (warp >= 4 && warp < 8) {
        // ------------------------------------------------------------------ GS transform warps
        const int r = (warp % 4) * 32 + lane;
        const int myhalf = r / kHalf;
        const uint32_t lane_off = (uint32_t)((warp % 4) * 32) << 16;
        const bool bf = p.in_dtype == DT_BF16;
        int s = 0, a = 0;
        uint32_t sph = 0, aph = 0;
        for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
            const ItemInfo I = decode_item(p, it);
            for (int t = I.t0; t < I.t1; ++t) {
                const int hv = tinfo_half(__ldg(p.sc.tinfo + t));
                const bool valid = (hv >> myhalf) & 1;
                mbar_wait(&s_full[s], sph);
                float rr = 1.f;
                if (GS) rr = valid ? reinterpret_cast<const float*>(smem + C::OFF_S + s * C::SB + C::XB + C::VB)[r] : 0.f;
                mbar_wait(&a_empty[a], aph ^ 1);
                tc_fence_after();
                const uint8_t* xs = smem + C::OFF_S + s * C::SB;
                const uint32_t a_tm = tmem_a + lane_off + a * (T / 2);
#pragma unroll 1
                for (int c = 0; c < T / 32; ++c) {  // 32 keys -> 16 packed words per step
                    uint32_t pk[16];
                    if (valid && rr != 0.f) {
#pragma unroll
                        for (int q4 = 0; q4 < 4; ++q4) {
                            const uint4 x = *reinterpret_cast<const uint4*>(xs + tile_chunk_off(r, c * 4 + q4));
                            const uint32_t xw[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
                            for (int u = 0; u < 4; ++u) {
                                if (GS) {  // Y = X' * r'  (fp16 X' -> fp32 -> x r' -> dtype)
                                    const float2 f = unpack_f16(xw[u]);
                                    pk[q4 * 4 + u] = bf ? pack_bf16(f.x * rr, f.y * rr) : pack_f16(f.x * rr, f.y * rr);
                                } else {   // P already holds dtype values
                                    pk[q4 * 4 + u] = xw[u];
                                }
                            }
                        }
                    } else {
#pragma unroll
                        for (int u = 0; u < 16; ++u) pk[u] = 0u;
                    }
                    tmem_st16(a_tm + c * 16, pk);
                }
                tmem_wait_st();
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&a_full[a]);
                if (++s == C::NS) { s = 0; sph ^= 1; }
                if (++a == C::NA) { a = 0; aph ^= 1; }
            }
        }
    } else if (warp >= 8) {
        // ------------------------------------------------------------------ output epilogue
        const int r = (warp % 4) * 32 + lane;
        const uint32_t lane_off = (uint32_t)((warp % 4) * 32) << 16;
        int o = 0;
        uint32_t oph = 0;
        for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
            const ItemInfo I = decode_item(p, it);
            const size_t orow = (size_t)I.g * p.S + I.rb * kRowBlock + r;
            if (I.t0 == I.t1) {  // no kept key anywhere in these rows: output 0 (reading R9)
                if (p.out_dtype == DT_F32) {
                    float4* O = reinterpret_cast<float4*>((float*)p.out + orow * D);
                    for (int c = 0; c < D / 4; ++c) O[c] = make_float4(0.f, 0.f, 0.f, 0.f);
                } else {
                    uint4* O = reinterpret_cast<uint4*>((uint16_t*)p.out + orow * D);
                    for (int c = 0; c < D / 8; ++c) O[c] = make_uint4(0, 0, 0, 0);
                }
                continue;
            }
            mbar_wait(&o_full[o], oph);
            tc_fence_after();
            const uint32_t taddr = tmem_o + lane_off + o * D;
#pragma unroll 1
            for (int c = 0; c < D / 32; ++c) {
                uint32_t v[32];
                tmem_ld32(taddr + c * 32, v);
                tmem_wait_ld();
                if (p.out_dtype == DT_F32) {
                    float4* O = reinterpret_cast<float4*>((float*)p.out + orow * D + c * 32);
#pragma unroll
                    for (int u = 0; u < 8; ++u)
                        O[u] = make_float4(__uint_as_float(v[4 * u]), __uint_as_float(v[4 * u + 1]),
                                           __uint_as_float(v[4 * u + 2]), __uint_as_float(v[4 * u + 3]));
                } else {
                    uint32_t pk[16];
#pragma unroll
                    for (int u = 0; u < 16; ++u) {
                        const float f0 = __uint_as_float(v[2 * u]), f1 = __uint_as_float(v[2 * u + 1]);
                        pk[u] = p.out_dtype == DT_BF16 ? pack_bf16(f0, f1) : pack_f16(f0, f1);
                    }
                    uint4* O = reinterpret_cast<uint4*>((uint16_t*)p.out + orow * D + c * 32);
#pragma unroll
                    for (int u = 0; u < 4; ++u) O[u] = make_uint4(pk[4 * u], pk[4 * u + 1], pk[4 * u + 2], pk[4 * u + 3]);
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&o_empty[o]);
            if (++o == C::NO) { o = 0; oph ^= 1; }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

// ============================================================================ unfused softmax
// One warp per query row (the paper's baseline keeps one row vector per TB in on-chip memory,
// PAPER.md L102): read the row's score pieces once into shared memory, max, sum, write P once.
template <int T>
__global__ void __launch_bounds__(128) row_softmax(const Params p)
{
    extern __shared__ uint32_t rowbuf[];  // per warp: S/2 words (fp16 pairs of this row)
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int64_t row = (int64_t)blockIdx.x * 4 + warp;
    if (row >= (int64_t)p.B * p.H * p.S) return;
    uint32_t* buf = rowbuf + (size_t)warp * (p.S / 2);
    const int g = (int)(row / p.S), i = (int)(row % p.S);
    const int rb = i / kRowBlock, r = i % kRowBlock, myhalf = r / kHalf;
    const DevSched& sc = p.sc;
    const int lh = lh_of(sc, g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    const int t0 = tp[rb], t1 = tp[rb + 1];
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - tp[0];
    constexpr int XB = kRowBlock * T * 2;
    // lane l reads 4 bytes (2 scores) at physical byte 4l of each 128-B row piece
    const int pchunk = lane / 4, within = lane % 4;
    const int lchunk = pchunk ^ (r & 7);
    float mx = -INFINITY;
    int nw = 0;
    for (int t = t0; t < t1; ++t) {
        if (!((tinfo_half(sc.tinfo[t]) >> myhalf) & 1)) continue;
        const uint8_t* tile = (const uint8_t*)p.xprime + (slot0 + t) * (int64_t)XB;
        for (int ch = 0; ch < T / 64; ++ch) {
            const uint32_t w = *reinterpret_cast<const uint32_t*>(tile + ch * (kRowBlock * 128) + r * 128 + lane * 4);
            buf[nw * 32 + lane] = w;
            const float2 f = unpack_f16(w);
            mx = fmaxf(mx, fmaxf(f.x, f.y));
            ++nw;
        }
    }
    for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    const float l2e = 1.4426950408889634f;
    const float neg = mx == -INFINITY ? 0.f : -mx * l2e;
    float sum = 0.f;
    for (int k = 0; k < nw; ++k) {
        const float2 f = unpack_f16(buf[k * 32 + lane]);
        sum += ex2(fmaf(f.x, l2e, neg)) + ex2(fmaf(f.y, l2e, neg));
    }
    for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
    const float inv = sum > 0.f ? 1.f / sum : 0.f;
    const bool bf = p.in_dtype == DT_BF16;
    int k = 0;
    for (int t = t0; t < t1; ++t) {
        if (!((tinfo_half(sc.tinfo[t]) >> myhalf) & 1)) continue;
        uint8_t* tile = (uint8_t*)p.pbuf + (slot0 + t) * (int64_t)XB;
        for (int ch = 0; ch < T / 64; ++ch, ++k) {
            const float2 f = unpack_f16(buf[k * 32 + lane]);
            const float y0 = ex2(fmaf(f.x, l2e, neg)) * inv, y1 = ex2(fmaf(f.y, l2e, neg)) * inv;
            *reinterpret_cast<uint32_t*>(tile + ch * (kRowBlock * 128) + r * 128 + lane * 4) =
                bf ? pack_bf16(y0, y1) : pack_f16(y0, y1);
        }
    }
    (void)lchunk;
    (void)within;
}

// ============================================================================ host side

namespace {

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn encode_fn()
{
    static EncodeTiledFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeTiledFn)f;
    });
    return fn;
}

// [rows][D] 16-bit row-major tensor, box {64 cols, box_rows}, 128-B swizzle
cudaError_t make_tmap(CUtensorMap* m, const void* base, int64_t rows, int D, int box_rows, int dtype)
{
    EncodeTiledFn fn = encode_fn();
    if (!fn) return cudaErrorNotSupported;
    cuuint64_t dims[2] = {(cuuint64_t)D, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)D * 2};
    cuuint32_t box[2] = {64, (cuuint32_t)box_rows};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = fn(m, dtype == DT_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2,
                    const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

int num_sms()
{
    int dev = 0, n = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    return n;
}

template <int D, int T, bool LS>
cudaError_t launch_g1(const Params& p, cudaStream_t st, int64_t* nl)
{
    using C = G1<D, T>;
    CUtensorMap tq, tk;
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    cudaError_t e;
    if ((e = make_tmap(&tq, p.q, rows, D, kRowBlock, p.in_dtype)) != cudaSuccess) return e;
    if ((e = make_tmap(&tk, p.k, rows, D, T, p.in_dtype)) != cudaSuccess) return e;
    auto kern = tc_gemm1<D, T, LS>;
    if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM)) != cudaSuccess) return e;
    const int grid = std::min(p.sc.n_items, num_sms());
    kern<<<grid, C::THREADS, C::SMEM, st>>>(tq, tk, p);
    ++*nl;
    return cudaGetLastError();
}

template <int D, int T, bool GS>
cudaError_t launch_g2(const Params& p, cudaStream_t st, int64_t* nl)
{
    using C = G2<D, T>;
    CUtensorMap tv;
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    cudaError_t e;
    if ((e = make_tmap(&tv, p.v, rows, D, T, p.in_dtype)) != cudaSuccess) return e;
    auto kern = tc_gemm2<D, T, GS>;
    if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM)) != cudaSuccess) return e;
    const int grid = std::min(p.sc.n_items, num_sms());
    kern<<<grid, C::THREADS, C::SMEM, st>>>(tv, p);
    ++*nl;
    return cudaGetLastError();
}

template <int T>
cudaError_t launch_softmax(const Params& p, cudaStream_t st, int64_t* nl)
{
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    const size_t sm = 4 * (size_t)p.S * 2;
    cudaError_t e = cudaFuncSetAttribute(row_softmax<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    row_softmax<T><<<(unsigned)((rows + 3) / 4), 128, sm, st>>>(p);
    ++*nl;
    return cudaGetLastError();
}

template <int D, int T>
cudaError_t fused_dt(const Params& p, cudaStream_t st, int64_t* nl)
{
    cudaError_t e = cudaSuccess;
    if ((p.stages & 1) && (e = launch_g1<D, T, true>(p, st, nl)) != cudaSuccess) return e;
    if ((p.stages & 2) && (e = launch_ir(p, st, nl)) != cudaSuccess) return e;
    if (p.stages & 4) e = launch_g2<D, T, true>(p, st, nl);
    return e;
}

template <int D, int T>
cudaError_t unfused_dt(const Params& p, cudaStream_t st, int64_t* nl)
{
    cudaError_t e = cudaSuccess;
    if ((p.stages & 1) && (e = launch_g1<D, T, false>(p, st, nl)) != cudaSuccess) return e;
    if ((p.stages & 2) && (e = launch_softmax<T>(p, st, nl)) != cudaSuccess) return e;
    if (p.stages & 4) e = launch_g2<D, T, false>(p, st, nl);
    return e;
}

}  // namespace

cudaError_t launch_tc_fused(const Params& p, cudaStream_t st, int64_t* nl)
{
    if (p.D == 64) return p.T == 64 ? fused_dt<64, 64>(p, st, nl) : fused_dt<64, 128>(p, st, nl);
    return p.T == 64 ? fused_dt<128, 64>(p, st, nl) : fused_dt<128, 128>(p, st, nl);
}

cudaError_t launch_tc_unfused(const Params& p, cudaStream_t st, int64_t* nl)
{
    if (p.S > 16384) return cudaErrorNotSupported;  // row buffer of the baseline softmax
    if (p.D == 64) return p.T == 64 ? unfused_dt<64, 64>(p, st, nl) : unfused_dt<64, 128>(p, st, nl);
    return p.T == 64 ? unfused_dt<128, 64>(p, st, nl) : unfused_dt<128, 128>(p, st, nl);
}

}  // namespace sr
