// k_gemm1.cu -- GEMM1 = Q K^T with scale + mask, and the Local Softmax (LS) sub-layer fused into
// its epilogue ("setting T of the LS kernel equal to the output tile width
// of the MatMul kernel, the LS kernel can be fused to its preceding MatMul kernel"; scale and mask
// fused as element-wise layers, L169).  LS=false builds the unfused baseline's GEMM1, which writes
// the scaled, masked score tile S instead (L171).
//
// Per 128-row x T-key tile, fp32 accumulator in TMEM:
//   m'  = max_j x_j                    (x = Q K^T * scale, masked to -inf)
//   X'  = e^{x - m'}  -> fp16 tile, written to HBM once (the only attention-matrix write)
//   d'  = sum_j X'_j                   (fp32)
// m', d' go to the workspace as fp32 [slot][128 rows].
//
// Warp roles (persistent CTA per SM, 384 threads):
//   warp 0      TMA producer: Q tile per item (double-buffered), K tiles (NK-stage ring)
//   warp 1      MMA issuer: tcgen05.mma kind::f16, D/16 MMAs of 128 x T x 16 per tile into one
//               of NACC TMEM accumulators; publishes a per-tile header (slot, rows, key tile,
//               half-valid bits, kv_len) next to the accumulator -- acc_full completes when both
//               the header arrive and the MMA commit have landed
//   warp 2      TMEM allocator (512 columns)
//   warps 4-11  two epilogue warpgroups taking alternate tiles: one tcgen05.ld of the whole row,
//               accumulator released immediately, mask (interval bits), max, ex2, sum, fp16 pack,
//               st.shared into a swizzled staging tile, one cp.async.bulk store per tile
#include "tc_common.cuh"

namespace sr {

using namespace ptx;

struct G1Hdr {  // per-accumulator tile header, written by the MMA warp
    int32_t slot_lo, slot_hi, i0, kvl, w, flags, pad0, pad1;
};
enum : int { HDR_TILE = 1, HDR_END = 2 };

template <int D, int T, int XPWMAX = 2>
struct G1 {
    static constexpr int QB = kRowBlock * D * 2;  // Q tile bytes
    static constexpr int KB = T * D * 2;          // K tile bytes
    static constexpr int XB = kRowBlock * T * 2;  // X'/S tile bytes
    static constexpr int NQ = 2;
    static constexpr int NACC = 512 / T;  // TMEM accumulators (4 for T=128, 8 for T=64)
    // staging buffers per epilogue warpgroup: 2 when shared memory allows, else 1
    static constexpr int XPW = (XPWMAX >= 2 && NQ * QB + 2 * KB + 4 * XB + 4096 <= kSmemMax) ? 2 : 1;
    static constexpr int NK_ = (kSmemMax - 4096 - NQ * QB - 2 * XPW * XB) / KB;
    static constexpr int NK = NK_ > 4 ? 4 : NK_;
    static_assert(NK >= 2, "smem budget");
    static constexpr int OFF_Q = 0;
    static constexpr int OFF_K = OFF_Q + NQ * QB;
    static constexpr int OFF_X = OFF_K + NK * KB;
    static constexpr int OFF_BAR = OFF_X + 2 * XPW * XB;
    static constexpr int NBAR = 2 * NQ + 2 * NK + 2 * NACC;
    static constexpr int OFF_HDR = OFF_BAR + NBAR * 8;
    static constexpr int OFF_TPTR = OFF_HDR + NACC * (int)sizeof(G1Hdr);
    static constexpr int SMEM_ = OFF_TPTR + 16 + 1024;  // + alignment slack
    static constexpr int SMEM = SMEM_ > 118 * 1024 ? SMEM_ : 118 * 1024;  // 1 CTA/SM (512 TMEM cols)
    static constexpr int THREADS = 384;
};

template <int D, int T, bool LS, int XPWMAX>
__global__ void __launch_bounds__(384, 1)
    tc_gemm1(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK, const Params p)
{
    using C = G1<D, T, XPWMAX>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint64_t* bars = (uint64_t*)(smem + C::OFF_BAR);
    uint64_t* q_full = bars;
    uint64_t* q_empty = q_full + C::NQ;
    uint64_t* k_full = q_empty + C::NQ;
    uint64_t* k_empty = k_full + C::NK;
    uint64_t* acc_full = k_empty + C::NK;
    uint64_t* acc_empty = acc_full + C::NACC;
    G1Hdr* hdr = (G1Hdr*)(smem + C::OFF_HDR);
    uint32_t* tmem_ptr = (uint32_t*)(smem + C::OFF_TPTR);

    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (threadIdx.x == 0) {
        for (int i = 0; i < C::NQ; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
        for (int i = 0; i < C::NK; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
        // acc_full: header arrive (MMA thread) + tcgen05.commit; acc_empty: one arrive per epilogue warp
        for (int i = 0; i < C::NACC; ++i) { mbar_init(&acc_full[i], 2); mbar_init(&acc_empty[i], 4); }
        fence_mbar_init();
    }
    if (warp == 0 && lane == 0) { prefetch_tmap(&tmQ); prefetch_tmap(&tmK); }
    if (warp == 2) tmem_alloc(tmem_ptr, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_ptr;
    // PDL: the prologue above overlapped the previous kernel's tail; let the next kernel start its
    // own prologue, then wait for our producer kernel's results before touching them
    griddep_launch_dependents();
    griddep_wait();
    const int n_items = p.sc.n_items;

    if (warp < 4) {
        // warpgroup 0 hands registers to the epilogue warpgroups (168/thread at launch)
        reg_dealloc<56>();
        if (warp == 0 && lane == 0) {
            // -------------------------------------------------------------- TMA producer
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
                int w_next = __ldg(p.sc.tinfo + I.t0);
                for (int t = I.t0; t < I.t1; ++t) {
                    const int w = w_next;
                    if (t + 1 < I.t1) w_next = __ldg(p.sc.tinfo + t + 1);
                    mbar_wait(&k_empty[ks], kph ^ 1);
                    mbar_arrive_expect_tx(&k_full[ks], C::KB);
                    for (int h = 0; h < D / 64; ++h)
                        tma_load_2d(smem + C::OFF_K + ks * C::KB + h * (T * 128), &tmK, h * 64,
                                    I.g * p.S + tinfo_kt(w) * T, &k_full[ks]);
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                }
            }
        } else if (warp == 1 && lane == 0) {
            // -------------------------------------------------------------- MMA issuer
            const uint32_t idesc = idesc_f16(p.in_dtype == DT_BF16 ? 1 : 0, kRowBlock, T, 0, 0);
            int qi = 0, ks = 0, n = 0;
            uint32_t qph = 0, kph = 0;
            for (int it = blockIdx.x; it < n_items; it += gridDim.x) {
                const ItemInfo I = decode_item(p, it);
                if (I.t0 == I.t1) continue;
                const int kvl = p.sc.kv_len ? __ldg(p.sc.kv_len + I.g / p.H) : p.S;
                mbar_wait(&q_full[qi], qph);
                tc_fence_after();
                const uint32_t q_addr = smem_u32(smem + C::OFF_Q + qi * C::QB);
                int w_next = __ldg(p.sc.tinfo + I.t0);
                for (int t = I.t0; t < I.t1; ++t, ++n) {
                    const int w = w_next;
                    if (t + 1 < I.t1) w_next = __ldg(p.sc.tinfo + t + 1);
                    const int ab = n % C::NACC;
                    mbar_wait(&acc_empty[ab], ((n / C::NACC) & 1) ^ 1);
                    const int64_t slot = I.slot0 + t;
                    hdr[ab] = G1Hdr{(int32_t)(slot & 0xffffffff), (int32_t)(slot >> 32), I.rb * kRowBlock, kvl, w,
                                    HDR_TILE, I.g, 0};
                    mbar_arrive(&acc_full[ab]);  // header published (arrival 1 of 2)
                    mbar_wait(&k_full[ks], kph);
                    tc_fence_after();
                    const uint32_t k_addr = smem_u32(smem + C::OFF_K + ks * C::KB);
                    const uint32_t d_tmem = tmem_base + ab * T;
#pragma unroll
                    for (int kk = 0; kk < D / 16; ++kk) {
                        const uint32_t h = kk / 4, wk = kk % 4;
                        const uint64_t ad = smem_desc_sw128(q_addr + h * (kRowBlock * 128) + wk * 32, 16, 1024);
                        const uint64_t bd = smem_desc_sw128(k_addr + h * (T * 128) + wk * 32, 16, 1024);
                        mma_ss(d_tmem, ad, bd, idesc, kk > 0 ? 1u : 0u);
                    }
                    mma_commit(&k_empty[ks]);
                    mma_commit(&acc_full[ab]);  // arrival 2 of 2 when the MMAs complete
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                }
                mma_commit(&q_empty[qi]);
                if (++qi == C::NQ) { qi = 0; qph ^= 1; }
            }
            for (int e = 0; e < 2; ++e, ++n) {  // one END header for each epilogue warpgroup
                const int ab = n % C::NACC;
                mbar_wait(&acc_empty[ab], ((n / C::NACC) & 1) ^ 1);
                hdr[ab].flags = HDR_END;
                mbar_arrive(&acc_full[ab]);
                mbar_arrive(&acc_full[ab]);
            }
        }
    } else {
        reg_alloc<224>();
        // ------------------------------------------------------------------ epilogue warpgroups
        const int e = (warp - 4) / 4;          // warpgroup 0 / 1: even / odd tiles
        const int r = (warp % 4) * 32 + lane;  // tile row == TMEM lane
        const int myhalf = r / kHalf;
        const uint32_t lane_off = (uint32_t)((warp % 4) * 32) << 16;
        const bool issuer = (threadIdx.x % 128) == 0;
        const float sl2 = p.scale_log2;
        int k = 0;  // tiles processed by this warpgroup
        for (int n = e;; n += 2, ++k) {
            const int buf = n % C::NACC;
            mbar_wait(&acc_full[buf], (uint32_t)(n / C::NACC) & 1);
            tc_fence_after();
            const G1Hdr H = hdr[buf];
            if (H.flags & HDR_END) break;
            const int kt = tinfo_kt(H.w), hv = tinfo_half(H.w);
            const bool valid = (hv >> myhalf) & 1;
            const int c0 = kt * T, i = H.i0 + r;
            const int64_t slot = ((int64_t)H.slot_hi << 32) | (uint32_t)H.slot_lo;
            // one TMEM read of the row's T fp32 scores; the accumulator goes straight back to the MMA
            uint32_t xr[T];
            if (valid) {
#pragma unroll
                for (int c = 0; c < T / 32; ++c)
                    tmem_ld32(tmem_base + lane_off + buf * T + c * 32, *reinterpret_cast<uint32_t(*)[32]>(&xr[c * 32]));
                tmem_wait_ld();
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&acc_empty[buf]);
            uint8_t* stage = smem + C::OFF_X + (e * C::XPW + (k % C::XPW)) * C::XB;
            const uint32_t stage_s = smem_u32(stage);
            // staging buffer free: this warpgroup's store from it (XPW tiles ago) has read it
            if (issuer) {
                if (C::XPW == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
                else bulk_wait_read0();
            }
            named_bar_sync(1 + e, 128);
            float mx = -INFINITY, dsum = 0.f;
            if (valid) {
                // mask layer: kept keys of this row form <= 2 intervals
                const RowMask rm = row_mask(p, i, H.kvl);
#pragma unroll
                for (int c = 0; c < T / 32; ++c) {
                    const uint32_t bits = mask_bits32(rm, c0 + c * 32);
                    if (bits != 0xffffffffu) {
#pragma unroll
                        for (int u = 0; u < 32; ++u)
                            if (!((bits >> u) & 1u)) xr[c * 32 + u] = 0xff800000u;  // -inf
                    }
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
                    // X' = e^{x - m'}: base 2 with log2(e) folded into the scale, one FFMA + one MUFU
                    neg = (mx == -INFINITY) ? 0.f : -mx * sl2;
                }
                float s4[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                for (int q4 = 0; q4 < T / 8; ++q4) {  // 8 keys -> one 16-B chunk of the tile
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
                    sts128(stage_s + tile_chunk_off(r, q4), w4[0], w4[1], w4[2], w4[3]);
                }
                dsum = (s4[0] + s4[1]) + (s4[2] + s4[3]);
            }
            fence_proxy_async_smem();
            named_bar_sync(1 + e, 128);
            if (issuer) {  // the tile's valid 64-row halves go to HBM in one or two bulk copies
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
        if (issuer) bulk_wait0();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

// ----------------------------------------------------------------------------- launchers

cudaError_t make_tmap_2d(CUtensorMap* m, const void* base, int64_t rows, int D, int box_rows, int dtype);
int num_sms();

template <int D, int T, bool LS>
cudaError_t launch_g1_t(const Params& p, cudaStream_t st, int64_t* nl)
{
    using C = G1<D, T, 2>;
    CUtensorMap tq, tk;
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    cudaError_t e;
    if ((e = make_tmap_2d(&tq, p.q, rows, D, kRowBlock, p.in_dtype)) != cudaSuccess) return e;
    if ((e = make_tmap_2d(&tk, p.k, rows, D, T, p.in_dtype)) != cudaSuccess) return e;
    auto kern = tc_gemm1<D, T, LS, 2>;
    if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM)) != cudaSuccess) return e;
    const int grid = std::min(p.sc.n_items, num_sms());
    return launch_pdl(kern, dim3(grid), dim3(C::THREADS), C::SMEM, st, nl, tq, tk, p);
}

cudaError_t launch_gemm1(const Params& p, bool ls, cudaStream_t st, int64_t* nl)
{
    if (p.D == 64) {
        if (p.T == 64) return ls ? launch_g1_t<64, 64, true>(p, st, nl) : launch_g1_t<64, 64, false>(p, st, nl);
        return ls ? launch_g1_t<64, 128, true>(p, st, nl) : launch_g1_t<64, 128, false>(p, st, nl);
    }
    if (p.T == 64) return ls ? launch_g1_t<128, 64, true>(p, st, nl) : launch_g1_t<128, 64, false>(p, st, nl);
    return ls ? launch_g1_t<128, 128, true>(p, st, nl) : launch_g1_t<128, 128, false>(p, st, nl);
}

}  // namespace sr
