// k_bwd.cu -- training backward of the softmax-recomposed attention layer (§6:
// "the derivative of the error is expressed as y, which means that the input of the softmax layer
// does not need to be stored").  The forward leaves the Local-Softmax tiles
// X' = e^{x - m'} (fp16), m' per (row, tile) and each row's (m, d) in the workspace; the backward
// recomposes y = X' r'_k (r'_k = e^{m'_k - m} / d, the Global Scaling of L151) tile by tile and
// never touches the score matrix x:
//
//   bwd_prep     per query row: m, 1/d (the two IR partials of GEMM1 merged), delta = dO . O
//   tc_bwd_ds    dP = dO V^T on the tensor cores (TMEM accumulator); epilogue, per element,
//                dS' = scale * y * (dP - delta) with y = X' r'  -- Eq. (3) in row form
//                (dE/dx_k = y_k (dE/dy_k - sum_i dE/dy_i y_i), sum_j y_ij dP_ij = dO_i . O_i) --
//                written in place over the X' stage and bulk-stored as a tile of the same slot;
//                r' of every (row, tile) goes to the workspace for the dV kernel
//   dQ           = dS' K: the GEMM2 kernel (k_gemm2.cu) in its plain mode, A = dS' tiles, B = K
//   tc_bwd_kv    per 128-key column block, over the row-blocks that list it (the transposed tile
//                schedule): dK = dS'^T Q (A = dS' tile read MN-major from smem) and, with PV,
//                dV = y^T dO (A = X' tile scaled by r' in place in smem, then read MN-major)
//
// Masked elements need no mask logic here: X' is exactly 0 there, so y, dS' and every
// contribution vanish; invalid 64-row halves of a tile (reading R22) are zero-filled or skipped.
#include "tc_common.cuh"

namespace sr {

using namespace ptx;

cudaError_t make_tmap_2d(CUtensorMap* m, const void* base, int64_t rows, int D, int box_rows, int dtype);
cudaError_t launch_gemm2(const Params& p, int mode, cudaStream_t st, int64_t* nl);

constexpr int kMWB = 128;  // macro tile width (keys per MMA step) of the backward kernels

// never written: the zero source of the bulk copies that fill absent tiles / invalid halves
__device__ __align__(128) uint8_t g_zero_half[kHalf * 128];

__device__ __forceinline__ float2 unpack16(uint32_t w, bool bf) { return bf ? unpack_bf16(w) : unpack_f16(w); }
__device__ __forceinline__ uint32_t pack16(float a, float b, bool bf) { return bf ? pack_bf16(a, b) : pack_f16(a, b); }

// ------------------------------------------------------------------------------ kernel 1
// bstat[0][row] = m, bstat[1][row] = 1/d (merged from GEMM1's two IR partials exactly as GEMM2's
// prologue merges them), bstat[2][row] = delta = sum_d dO[row, d] * O[row, d].  D/8 threads per
// row for the dot product (16 B of dO each), then one thread per row for the statistics.
constexpr int kPrepThreads = 512;
#ifndef SR_PREP_TPR
#define SR_PREP_TPR 8  // threads per row of bwd_prep (measured on C3: 8 -> 16 us, 16 -> 23 us, 4 -> 21 us)
#endif

template <int D>
__global__ void __launch_bounds__(kPrepThreads) bwd_prep(const Params p)
{
    griddep_launch_dependents();
    griddep_wait();
    constexpr int TPR = SR_PREP_TPR;           // threads per row
    constexpr int EPT = D / TPR;               // elements per thread (16-B loads of 8)
    constexpr int RPB = kPrepThreads / TPR;    // rows per block
    __shared__ float s_delta[RPB];
    const int64_t nrow = (int64_t)p.B * p.H * p.S;
    const int64_t row0 = (int64_t)blockIdx.x * RPB;
    const int64_t row = row0 + threadIdx.x / TPR;
    const int c = threadIdx.x % TPR;
    // the statistics threads issue their IR-partial loads first, so the two memory round trips of a
    // block (dO / O, then rowstat) overlap instead of running back to back
    const int64_t rs = row0 + threadIdx.x;
    // rowstat / bstat rows are laid out per head in whole row-blocks (p.Spad): the row's index there
    const int64_t nrowp = (int64_t)p.B * p.H * p.Spad, rsp = (rs / p.S) * p.Spad + rs % p.S;
    float ma = -INFINITY, da = 0.f, mb = -INFINITY, db = 0.f;
    if (threadIdx.x < RPB && rs < nrow) {
        ma = __ldcg(p.rowstat + rsp);
        da = __ldcg(p.rowstat + nrowp + rsp);
        mb = __ldcg(p.rowstat + 2 * nrowp + rsp);
        db = __ldcg(p.rowstat + 3 * nrowp + rsp);
    }
    float acc = 0.f;
    if (row < nrow) {
        const bool bf = p.in_dtype == DT_BF16;
        uint4 g[EPT / 8], o16[EPT / 8];
        float4 o32[EPT / 4];
#pragma unroll
        for (int k = 0; k < EPT / 8; ++k)  // chunk c + k * TPR of the row: coalesced across the row's threads
            g[k] = __ldcg(reinterpret_cast<const uint4*>((const uint16_t*)p.dout + row * D) + c + k * TPR);
        if (p.out_dtype == DT_F32) {
#pragma unroll
            for (int k = 0; k < EPT / 8; ++k) {
                const float4* o4 = reinterpret_cast<const float4*>((const float*)p.out + row * D) + 2 * (c + k * TPR);
                o32[2 * k] = __ldcg(o4);
                o32[2 * k + 1] = __ldcg(o4 + 1);
            }
        } else {
#pragma unroll
            for (int k = 0; k < EPT / 8; ++k)
                o16[k] = __ldcg(reinterpret_cast<const uint4*>((const uint16_t*)p.out + row * D) + c + k * TPR);
        }
#pragma unroll
        for (int k = 0; k < EPT / 8; ++k) {
            const uint32_t gw[4] = {g[k].x, g[k].y, g[k].z, g[k].w};
            float od[8];
            if (p.out_dtype == DT_F32) {
                const float4 a = o32[2 * k], b = o32[2 * k + 1];
                od[0] = a.x; od[1] = a.y; od[2] = a.z; od[3] = a.w; od[4] = b.x; od[5] = b.y; od[6] = b.z; od[7] = b.w;
            } else {
                const uint32_t ow[4] = {o16[k].x, o16[k].y, o16[k].z, o16[k].w};
#pragma unroll
                for (int w = 0; w < 4; ++w) {
                    const float2 f = unpack16(ow[w], p.out_dtype == DT_BF16);
                    od[2 * w] = f.x;
                    od[2 * w + 1] = f.y;
                }
            }
#pragma unroll
            for (int w = 0; w < 4; ++w) {
                const float2 f = unpack16(gw[w], bf);
                acc = fmaf(f.x, od[2 * w], acc);
                acc = fmaf(f.y, od[2 * w + 1], acc);
            }
        }
    }
#pragma unroll
    for (int o = TPR / 2; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (c == 0) s_delta[threadIdx.x / TPR] = acc;
    __syncthreads();
    // per-row statistics with one thread per row: coalesced loads of the IR partials and stores
    if (threadIdx.x < RPB && rs < nrow) {
        const int64_t r = rs;
        const float m = fmaxf(ma, mb);  // m = max_w m_w, d = sum_w e^{m_w - m} d_w
        const float d = m == -INFINITY ? 0.f : da * __expf(ma - m) + db * __expf(mb - m);
        p.bstat[rsp] = m;
        p.bstat[nrowp + rsp] = d > 0.f ? 1.f / d : 0.f;
        p.bstat[2 * nrowp + rsp] = s_delta[threadIdx.x];
        if (p.bwd_dq_fused) {  // dQ of a row-block with no listed tile is 0 (the dS' kernel never visits it)
            const int g = (int)(r / p.S), rb = (int)((r % p.S) / kRowBlock);
            const int32_t* tp = p.sc.tp + (size_t)lh_of(p.sc, g, p.H) * (p.sc.n_rb + 1);
            if (__ldcg(tp + rb + 1) == __ldcg(tp + rb)) {
                if (p.out_dtype == DT_F32) {
                    float4* O = reinterpret_cast<float4*>((float*)p.dq + r * D);
                    for (int c = 0; c < D / 4; ++c) O[c] = make_float4(0.f, 0.f, 0.f, 0.f);
                } else {
                    uint4* O = reinterpret_cast<uint4*>((uint16_t*)p.dq + r * D);
                    for (int c = 0; c < D / 8; ++c) O[c] = make_uint4(0, 0, 0, 0);
                }
            }
        }
    }
}

// ------------------------------------------------------------------------------ kernel 2
struct BHdr {  // per-accumulator macro-tile header (MMA warp -> epilogue)
    int32_t slot_lo, slot_hi, row_lo, row_hi, w0, w1, flags, pad;
};
enum : int { BH_TILE = 1, BH_END = 2, BH_LAST = 4 };

// DQ: dQ = dS' K is accumulated in TMEM inside this kernel (a CTA owns whole rows): after the
// epilogue has written a macro tile's dS' in place, the MMA warp multiplies that shared-memory
// tile (K-major A operand) by the tile's K rows (MN-major B, own ring loaded by warp 2); the
// epilogue warpgroup that finished the item's last tile writes the item's dQ rows.  Saves the
// separate dQ kernel's full re-read of dS'.
template <int D, bool DQ = false>
struct BD {
    static constexpr int QB = kRowBlock * D * 2;     // dO tile of a row-block
    static constexpr int KB = kMWB * D * 2;          // V stage (128 keys); also a K stage (DQ)
    static constexpr int XB = kRowBlock * kMWB * 2;  // X' (then dS') macro tile
    static constexpr int XSB = XB + 2048;            // + m' (2 x 512 B) + slack (1 KB aligned)
    static constexpr int NQ = (D == 64 && !DQ) ? 2 : 1;
    static constexpr int NK = (D == 64 && !DQ) ? 3 : 2;
    static constexpr int NKQ = DQ ? (D == 64 ? 2 : 1) : 0;  // K ring of the dQ MMA
    // X' stages: one ring per epilogue warpgroup (macro tile n -> warpgroup n % 2, its stage
    // (n / 2) % NXW).  A ring shared by both warpgroups would let one of them wait on a stage two
    // phases ahead of the other (an mbarrier parity wait cannot tell those phases apart).
    static constexpr int NX_ = (kSmemMax - 4096 - NQ * QB - (NK + NKQ) * KB) / XSB;
    static constexpr int NX = NX_ >= 4 ? 4 : 2;
    static_assert(NX_ >= 2, "smem budget");
    static constexpr int NXW = NX / 2;
    static constexpr int NACC = DQ ? 2 : 512 / kMWB;  // dP accumulators (DQ: + 2 x D columns of dQ)
    static constexpr int OFF_Q = 0;
    static constexpr int OFF_K = OFF_Q + NQ * QB;
    static constexpr int OFF_KQ = OFF_K + NK * KB;
    static constexpr int OFF_X = OFF_KQ + NKQ * KB;
    static constexpr int OFF_BAR = OFF_X + NX * XSB;
    // + DQ: kq_full / kq_empty, ds_ready per X' stage, dq_full / dq_empty
    static constexpr int NBAR = 2 * NQ + 2 * NK + 2 * NX + 2 * NACC + 2 * NKQ + NX + 4;
    static constexpr int OFF_HDR = OFF_BAR + NBAR * 8;
    static constexpr int OFF_TPTR = OFF_HDR + (NACC + 2) * (int)sizeof(BHdr);
    static constexpr int SMEM = OFF_TPTR + 16 + 1024;
    static_assert(SMEM <= kSmemMax, "smem budget");
    static constexpr int THREADS = 384;
};

template <int D, int T, bool DQ>
__global__ void __launch_bounds__(384, 1)
    tc_bwd_ds(const __grid_constant__ CUtensorMap tmO, const __grid_constant__ CUtensorMap tmV,
              const __grid_constant__ CUtensorMap tmK, const Params p)
{
    using C = BD<D, DQ>;
    constexpr int NSUB = kMWB / T;
    constexpr int XS = kRowBlock * T * 2;  // slot bytes (sub-tile)
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint64_t* bars = (uint64_t*)(smem + C::OFF_BAR);
    uint64_t* q_full = bars;
    uint64_t* q_empty = q_full + C::NQ;
    uint64_t* k_full = q_empty + C::NQ;
    uint64_t* k_empty = k_full + C::NK;
    uint64_t* x_full = k_empty + C::NK;
    uint64_t* x_empty = x_full + C::NX;
    uint64_t* acc_full = x_empty + C::NX;
    uint64_t* acc_empty = acc_full + C::NACC;
    uint64_t* kq_full = acc_empty + C::NACC;  // DQ
    uint64_t* kq_empty = kq_full + C::NKQ;
    uint64_t* ds_ready = kq_empty + C::NKQ;
    uint64_t* dq_full = ds_ready + C::NX;
    uint64_t* dq_empty = dq_full + 2;
    BHdr* hdr = (BHdr*)(smem + C::OFF_HDR);
    BHdr* dqhdr = hdr + C::NACC;
    uint32_t* tmem_ptr = (uint32_t*)(smem + C::OFF_TPTR);

    const int warp = warp_uniform(), lane = threadIdx.x % 32;
    if (threadIdx.x == 0) {
        for (int i = 0; i < C::NQ; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
        for (int i = 0; i < C::NK; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
        // x_empty: the epilogue warps once their bulk store has read the dS' (+ the dQ MMA commit)
        for (int i = 0; i < C::NX; ++i) { mbar_init(&x_full[i], 1); mbar_init(&x_empty[i], DQ ? 5 : 4); }
        for (int i = 0; i < C::NACC; ++i) { mbar_init(&acc_full[i], 2); mbar_init(&acc_empty[i], 4); }
        for (int i = 0; i < C::NKQ; ++i) { mbar_init(&kq_full[i], 1); mbar_init(&kq_empty[i], 1); }
        if (DQ) {
            for (int i = 0; i < C::NX; ++i) mbar_init(&ds_ready[i], 4);
            for (int i = 0; i < 2; ++i) { mbar_init(&dq_full[i], 2); mbar_init(&dq_empty[i], 4); }
        }
        fence_mbar_init();
    }
    if (warp == 0 && lane == 0) { prefetch_tmap(&tmO); prefetch_tmap(&tmV); if (DQ) prefetch_tmap(&tmK); }
    if (warp == 2) tmem_alloc(tmem_ptr, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_ptr;
    griddep_launch_dependents();
    griddep_wait();
    const int it_begin = __ldcg(p.sc.cta_ptr + blockIdx.x), it_end = __ldcg(p.sc.cta_ptr + blockIdx.x + 1);

    if (warp < 4) {
        reg_dealloc<56>();  // 4 warps x 32 x (168 - 56) = 8 warps x 32 x (224 - 168)
        if (warp == 0) {
            // ------------------------------------------------------------------ dO + V producer
            const uint64_t pol_v = policy_evict_last();  // V is re-read by every row-block of its head
            int qi = 0, ks = 0;
            uint32_t qph = 0, kph = 0;
            for (ItemWalk iw(p.sc, it_begin, it_end); iw.more();) {
                const ItemInfo I = iw.next();
                if (I.t0 == I.t1) continue;
                mbar_wait(&q_empty[qi], qph ^ 1);
                if (elect_one()) {
                    mbar_arrive_expect_tx(&q_full[qi], C::QB);
                    for (int h = 0; h < D / 64; ++h)
                        tma_load_2d(smem + C::OFF_Q + qi * C::QB + h * (kRowBlock * 128), &tmO, h * 64,
                                    I.g * p.S + I.rb * kRowBlock, &q_full[qi]);
                }
                __syncwarp();
                if (++qi == C::NQ) { qi = 0; qph ^= 1; }
                for (int t = I.t0; t < I.t1; t += NSUB) {
                    const int nsub = min(NSUB, I.t1 - t);
                    int w[NSUB];
#pragma unroll
                    for (int s = 0; s < NSUB; ++s) w[s] = s < nsub ? __ldcg(p.sc.tinfo + t + s) : 0;
                    mbar_wait(&k_empty[ks], kph ^ 1);
                    if (elect_one()) {
                        mbar_arrive_expect_tx(&k_full[ks], nsub * T * D * 2);
                        for (int s = 0; s < nsub; ++s)
                            for (int h = 0; h < D / 64; ++h)
                                tma_load_2d_hint(smem + C::OFF_K + ks * C::KB + h * (kMWB * 128) + s * (T * 128), &tmV,
                                                 h * 64, I.g * p.S + tinfo_kt(w[s]) * T, &k_full[ks], pol_v);
                    }
                    __syncwarp();
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                }
            }
        } else if (DQ && warp == 2) {
            // ------------------------------------------------------------------ K producer (dQ)
            const uint64_t pol_k = policy_evict_last();  // K is re-read by every row-block of its head
            int ks = 0;
            uint32_t kph = 0;
            for (ItemWalk iw(p.sc, it_begin, it_end); iw.more();) {
                const ItemInfo I = iw.next();
                for (int t = I.t0; t < I.t1; t += NSUB) {
                    const int nsub = min(NSUB, I.t1 - t);
                    int w[NSUB];
#pragma unroll
                    for (int s = 0; s < NSUB; ++s) w[s] = s < nsub ? __ldcg(p.sc.tinfo + t + s) : 0;
                    mbar_wait(&kq_empty[ks], kph ^ 1);
                    if (elect_one()) {
                        mbar_arrive_expect_tx(&kq_full[ks], nsub * T * D * 2);
                        for (int s = 0; s < nsub; ++s)
                            for (int h = 0; h < D / 64; ++h)
                                tma_load_2d_hint(smem + C::OFF_KQ + ks * C::KB + h * (kMWB * 128) + s * (T * 128), &tmK,
                                                 h * 64, I.g * p.S + tinfo_kt(w[s]) * T, &kq_full[ks], pol_k);
                    }
                    __syncwarp();
                    if (++ks == C::NKQ) { ks = 0; kph ^= 1; }
                }
            }
        } else if (warp == 3) {
            // ------------------------------------------------------------------ X' + m' producer
            // X' is streamed (evict_first) unless X' and dS' together fit in 0.8 of the L2 (p.x_evict_first)
            const uint64_t pol_x = p.x_evict_first ? policy_evict_first() : policy_evict_normal();
            int n = 0;  // macro tile counter, as the MMA warp and the epilogue count them
            for (ItemWalk iw(p.sc, it_begin, it_end); iw.more();) {
                const ItemInfo I = iw.next();
                for (int t = I.t0; t < I.t1; t += NSUB) {
                    const int nsub = min(NSUB, I.t1 - t);
                    int hv[NSUB];
                    uint32_t bytes = 0;
#pragma unroll
                    for (int u = 0; u < NSUB; ++u) {
                        hv[u] = u < nsub ? tinfo_half(__ldcg(p.sc.tinfo + t + u)) : 0;
                        if (u < nsub) bytes += (hv[u] == 3 ? 2 : 1) * (T / 64) * (kHalf * 128) + kRowBlock * 4;
                    }
                    const int xs = (n % 2) * C::NXW + (n / 2) % C::NXW;
                    const uint32_t xph = (uint32_t)((n / 2) / C::NXW) & 1;
                    mbar_wait(&x_empty[xs], xph ^ 1);
                    uint8_t* st = smem + C::OFF_X + xs * C::XSB;
                    if (elect_one()) {
                        mbar_arrive_expect_tx(&x_full[xs], bytes);
                        const uint8_t* src = (const uint8_t*)p.xprime + (I.slot0 + t) * (int64_t)XS;
                        for (int u = 0; u < nsub; ++u) {
                            for (int ch = 0; ch < T / 64; ++ch) {
                                const int o = u * XS + ch * (kRowBlock * 128);
                                if (hv[u] == 3) bulk_load_hint(st + o, src + o, kRowBlock * 128, &x_full[xs], pol_x);
                                else {
                                    const int o2 = o + (hv[u] == 2 ? kHalf * 128 : 0);
                                    bulk_load_hint(st + o2, src + o2, kHalf * 128, &x_full[xs], pol_x);
                                }
                            }
                            bulk_load(st + C::XB + u * 512, p.mprime + (I.slot0 + t + u) * kRowBlock, kRowBlock * 4,
                                      &x_full[xs]);
                        }
                    }
                    __syncwarp();
                    ++n;
                }
            }
        } else if (warp == 1) {
            // ------------------------------------------------------------------ MMA: dP = dO V^T
            // (DQ: then, one macro tile behind, dQ += dS' K once the epilogue has written the dS')
            const uint32_t idesc = idesc_f16(p.in_dtype == DT_BF16 ? 1 : 0, kRowBlock, kMWB, 0, 0);
            const uint32_t idesc_q = idesc_f16(p.in_dtype == DT_BF16 ? 1 : 0, kRowBlock, D, 0, 1);
            int qi = 0, ks = 0, n = 0;
            uint32_t qph = 0, kph = 0;
            // the pending dQ step: macro tile pn (-1: none), its sub-tile count, item flags and rows
            int pn = -1, pnsub = 0, pfirst = 0, plast = 0, pitem = 0, qs = 0, nitem = 0;
            uint32_t qsph = 0;
            int64_t prow0 = 0;
            auto dq_step = [&]() {
                if (!DQ || pn < 0) return;
                const int sx = (pn % 2) * C::NXW + (pn / 2) % C::NXW;
                const int b = pitem & 1;  // the pending tile's item: dQ accumulator buffer
                mbar_wait(&ds_ready[sx], (uint32_t)((pn / 2) / C::NXW) & 1);
                mbar_wait(&kq_full[qs], qsph);
                if (pfirst) mbar_wait(&dq_empty[b], ((uint32_t)(pitem >> 1) & 1) ^ 1);
                tc_fence_after();
                const uint32_t x_addr = smem_u32(smem + C::OFF_X + sx * C::XSB);
                const uint32_t k_addr = smem_u32(smem + C::OFF_KQ + qs * C::KB);
                if (elect_one()) {
                    for (int kk = 0; kk < pnsub * (T / 16); ++kk) {
                        const uint64_t ad = smem_desc_sw128(x_addr + (kk / 4) * (kRowBlock * 128) + (kk % 4) * 32, 16, 1024);
                        const uint64_t bd = smem_desc_sw128(k_addr + kk * 2048, kMWB * 128, 1024);
                        mma_ss(tmem_base + C::NACC * kMWB + b * D, ad, bd, idesc_q, (pfirst && kk == 0) ? 0u : 1u);
                    }
                    mma_commit(&kq_empty[qs]);
                    mma_commit(&x_empty[sx]);
                    if (plast) {
                        dqhdr[b] = BHdr{0, 0, (int32_t)(prow0 & 0xffffffff), (int32_t)(prow0 >> 32), 0, 0, BH_TILE, 0};
                        mbar_arrive(&dq_full[b]);  // header (arrival 1 of 2)
                        mma_commit(&dq_full[b]);   // the item's dQ is complete (arrival 2 of 2)
                    }
                }
                __syncwarp();
                if (++qs == C::NKQ) { qs = 0; qsph ^= 1; }
                pn = -1;
            };
            for (ItemWalk iw(p.sc, it_begin, it_end); iw.more();) {
                const ItemInfo I = iw.next();
                if (I.t0 == I.t1) continue;
                const int64_t row0 = (int64_t)I.g * p.S + I.rb * kRowBlock;
                mbar_wait(&q_full[qi], qph);
                tc_fence_after();
                const uint32_t q_addr = smem_u32(smem + C::OFF_Q + qi * C::QB);
                ++nitem;
                for (int t = I.t0; t < I.t1; t += NSUB, ++n) {
                    const int w0 = __ldcg(p.sc.tinfo + t);
                    const int w1 = (NSUB > 1 && t + 1 < I.t1) ? __ldcg(p.sc.tinfo + t + 1) : -1;
                    const int ab = n % C::NACC;
                    mbar_wait(&acc_empty[ab], ((n / C::NACC) & 1) ^ 1);
                    const int64_t slot = I.slot0 + t;
                    const bool last = t + NSUB >= I.t1;
                    if (elect_one()) {
                        hdr[ab] = BHdr{(int32_t)(slot & 0xffffffff), (int32_t)(slot >> 32), (int32_t)(row0 & 0xffffffff),
                                       (int32_t)(row0 >> 32), w0, w1, BH_TILE | (last ? BH_LAST : 0), nitem - 1};
                        mbar_arrive(&acc_full[ab]);  // header published (arrival 1 of 2)
                    }
                    __syncwarp();
                    mbar_wait(&k_full[ks], kph);
                    tc_fence_after();
                    const uint32_t k_addr = smem_u32(smem + C::OFF_K + ks * C::KB);
                    const uint32_t d_tmem = tmem_base + ab * kMWB;
                    if (elect_one()) {
#pragma unroll
                        for (int kk = 0; kk < D / 16; ++kk) {
                            const uint32_t h = kk / 4, wk = kk % 4;
                            const uint64_t ad = smem_desc_sw128(q_addr + h * (kRowBlock * 128) + wk * 32, 16, 1024);
                            const uint64_t bd = smem_desc_sw128(k_addr + h * (kMWB * 128) + wk * 32, 16, 1024);
                            mma_ss(d_tmem, ad, bd, idesc, kk > 0 ? 1u : 0u);
                        }
                        mma_commit(&k_empty[ks]);
                        mma_commit(&acc_full[ab]);  // arrival 2 of 2
                    }
                    __syncwarp();
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                    dq_step();  // the previous macro tile's dQ (its dS' is being / has been written)
                    if (DQ) {
                        pn = n;
                        pnsub = min(NSUB, I.t1 - t);
                        pfirst = t == I.t0;
                        plast = last;
                        prow0 = row0;
                        pitem = nitem - 1;
                    }
                }
                if (elect_one()) mma_commit(&q_empty[qi]);
                __syncwarp();
                if (++qi == C::NQ) { qi = 0; qph ^= 1; }
            }
            dq_step();  // the last macro tile's dQ
            for (int e = 0; e < 2; ++e, ++n) {  // one END header per epilogue warpgroup
                const int ab = n % C::NACC;
                mbar_wait(&acc_empty[ab], ((n / C::NACC) & 1) ^ 1);
                if (elect_one()) {
                    hdr[ab].flags = BH_END;
                    mbar_arrive(&acc_full[ab]);
                    mbar_arrive(&acc_full[ab]);
                }
                __syncwarp();
            }
        }
    } else {
        reg_alloc<224>();
        // ---------------------------------------------------------------------- epilogue: Eq. (3)
        const int e = (warp - 4) / 4;          // warpgroup 0 / 1: even / odd macro tiles
        const int r = (warp % 4) * 32 + lane;  // tile row == TMEM lane
        const int myhalf = r / kHalf;
        const uint32_t lane_off = (uint32_t)((warp % 4) * 32) << 16;
        const int wrow0 = (warp % 4) * 32;
        const bool bf = p.in_dtype == DT_BF16;
        const int64_t nrow = (int64_t)p.B * p.H * p.Spad;
        const uint64_t pol_ds = p.x_evict_first ? policy_evict_first() : policy_evict_normal();
        int64_t cur = -1;
        float m_row = 0.f, invd_row = 0.f, delta_row = 0.f;
        for (int n = e;; n += 2) {
            const int buf = n % C::NACC;
            mbar_wait(&acc_full[buf], (uint32_t)(n / C::NACC) & 1);
            tc_fence_after();
            const BHdr Hd = lds_hdr(hdr + buf);
            if (Hd.flags & BH_END) break;
            const int wsub[2] = {Hd.w0, Hd.w1};
            bool vs[NSUB];
            bool any = false;
#pragma unroll
            for (int s = 0; s < NSUB; ++s) {
                vs[s] = wsub[s] != -1 && ((tinfo_half(wsub[s]) >> myhalf) & 1);
                any |= vs[s];
            }
            const int64_t row0 = ((int64_t)Hd.row_hi << 32) | (uint32_t)Hd.row_lo;
            const int64_t slot = ((int64_t)Hd.slot_hi << 32) | (uint32_t)Hd.slot_lo;
            if (row0 != cur) {  // a new row-block: this row's m, 1/d, delta (bstat rows per head in whole
                cur = row0;     // row-blocks, p.Spad)
                const int64_t prow = (row0 / p.S) * p.Spad + row0 % p.S + r;
                m_row = __ldcg(p.bstat + prow);
                invd_row = __ldcg(p.bstat + nrow + prow);
                delta_row = __ldcg(p.bstat + 2 * nrow + prow);
            }
            uint32_t xr[kMWB];  // dP of this row, fp32
            if (any) {
#pragma unroll
                for (int c = 0; c < kMWB / 32; ++c)
                    tmem_ld32(tmem_base + lane_off + buf * kMWB + c * 32, *reinterpret_cast<uint32_t(*)[32]>(&xr[c * 32]));
                tmem_wait_ld();
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&acc_empty[buf]);
            const int sx = e * C::NXW + (n / 2) % C::NXW;
            mbar_wait(&x_full[sx], (uint32_t)((n / 2) / C::NXW) & 1);
            uint8_t* stage = smem + C::OFF_X + sx * C::XSB;
            const uint32_t stage_s = smem_u32(stage);
#pragma unroll
            for (int s = 0; s < NSUB; ++s) {
                if (!vs[s]) {
                    if (DQ && wsub[s] != -1)  // rows of an invalid half: zeros, the dQ MMA reads every row
#pragma unroll
                        for (int q4 = 0; q4 < T / 8; ++q4) sts128(stage_s + tile_chunk_off(r, s * (T / 8) + q4), 0u, 0u, 0u, 0u);
                    continue;
                }
                const float mp = lds_f32(stage_s + C::XB + s * 512 + 4 * r);
                // r'_k = e^{m'_k - m} / d (Global Scaling); 0 for a masked sub-vector
                const float rr = (mp == -INFINITY) ? 0.f : __expf(mp - m_row) * invd_row;
                p.rprime[(slot + s) * kRowBlock + r] = rr;
                const float sc = p.scale * rr;
#pragma unroll
                for (int q4 = 0; q4 < T / 8; ++q4) {  // 8 keys per 16-B chunk, in place
                    const uint32_t off = tile_chunk_off(r, s * (T / 8) + q4);
                    const uint4 xv = lds128(stage_s + off);
                    const uint32_t xw[4] = {xv.x, xv.y, xv.z, xv.w};
                    uint32_t pk[4];
#pragma unroll
                    for (int w = 0; w < 4; ++w) {
                        const float2 f = unpack_f16(xw[w]);  // X'
                        const int u = s * T + q4 * 8 + 2 * w;
                        // dS' = scale * (X' r') * (dP - delta)
                        const float g0 = (__uint_as_float(xr[u]) - delta_row) * sc;
                        const float g1 = (__uint_as_float(xr[u + 1]) - delta_row) * sc;
                        pk[w] = pack16(f.x * g0, f.y * g1, bf);
                    }
                    sts128(stage_s + off, pk[0], pk[1], pk[2], pk[3]);
                }
            }
            bool wv[NSUB];
#pragma unroll
            for (int s = 0; s < NSUB; ++s) wv[s] = __shfl_sync(0xffffffffu, vs[s] ? 1 : 0, 0) != 0;
            fence_proxy_async_smem();
            __syncwarp();
            if (DQ && lane == 0) mbar_arrive(&ds_ready[sx]);  // the dS' tile is ready for the dQ MMA
            if (lane == 0) {
#pragma unroll
                for (int s = 0; s < NSUB; ++s) {
                    if (!wv[s]) continue;  // a warp's 32 rows lie in one 64-row half
                    uint8_t* dst = (uint8_t*)p.dsbuf + (slot + s) * (int64_t)XS;
                    for (int ch = 0; ch < T / 64; ++ch)
                        // evict_first: dS' (as large as X') is re-read only by the next kernel; keep
                        // the L2 for the V / K tiles every row-block of the head re-reads
                        bulk_store_hint(dst + ch * (kRowBlock * 128) + wrow0 * 128,
                                        stage + (s * (T / 64) + ch) * (kRowBlock * 128) + wrow0 * 128, 32 * 128, pol_ds);
                }
                bulk_commit();
                bulk_wait_read0();  // the stage is recycled once the store has read it
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&x_empty[sx]);
            if (DQ && (Hd.flags & BH_LAST)) {  // the item's dQ rows: TMEM -> out dtype -> global
                const int b = Hd.pad & 1;
                mbar_wait(&dq_full[b], (uint32_t)(Hd.pad >> 1) & 1);
                tc_fence_after();
                const BHdr qh = lds_hdr(dqhdr + b);
                const int64_t qrow0 = ((int64_t)qh.row_hi << 32) | (uint32_t)qh.row_lo, qrow = qrow0 + r;
                const bool inhead = qrow0 % p.S + r < p.S;  // S % 128 == 64: the last block's upper half is outside
                const uint32_t taddr = tmem_base + lane_off + C::NACC * kMWB + b * D;
#pragma unroll
                for (int c = 0; c < D / 32; ++c) {
                    uint32_t v[32];
                    tmem_ld32(taddr + c * 32, v);
                    tmem_wait_ld();
                    if (!inhead) {
                    } else if (p.out_dtype == DT_F32) {
                        float4* O = reinterpret_cast<float4*>((float*)p.dq + qrow * D + c * 32);
#pragma unroll
                        for (int u = 0; u < 8; ++u)
                            O[u] = make_float4(__uint_as_float(v[4 * u]), __uint_as_float(v[4 * u + 1]),
                                               __uint_as_float(v[4 * u + 2]), __uint_as_float(v[4 * u + 3]));
                    } else {
                        uint32_t pk[16];
#pragma unroll
                        for (int u = 0; u < 16; ++u)
                            pk[u] = pack16(__uint_as_float(v[2 * u]), __uint_as_float(v[2 * u + 1]), p.out_dtype == DT_BF16);
                        uint4* O = reinterpret_cast<uint4*>((uint16_t*)p.dq + qrow * D + c * 32);
#pragma unroll
                        for (int u = 0; u < 4; ++u) O[u] = make_uint4(pk[4 * u], pk[4 * u + 1], pk[4 * u + 2], pk[4 * u + 3]);
                    }
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&dq_empty[b]);
            }
        }
        if (lane == 0) bulk_wait0();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

// ------------------------------------------------------------------------------ kernel 4
enum : int { KV_TILE = 1, KV_END = 2, KV_EMPTY = 4 };
struct KHdr {  // stage header (producer -> transform) / accumulator header (MMA -> epilogue)
    int32_t flags, hv0, hv1, pad0, row_lo, row_hi, pad1, pad2;
};

template <int D, bool PAIRED = (D == 64)>
struct BK {
    static constexpr int AB = kRowBlock * kMWB * 2;  // A: [2 key chunks of 64][128 rows][64] = 32 KB
    static constexpr int BB = kRowBlock * D * 2;     // B: Q (dK) or dO (dV) rows of the row-block
    static constexpr int SB = AB + BB + 2048;        // + r' (2 x 512 B) + header, 1 KB aligned
    // PAIRED (D = 64, dense / window layouts): two stages, so that a dV CTA and a dK CTA fit on one
    // SM together (smem < 113 KB, TMEM 128 columns each) and overlap each other's latencies
    // (measured: C2 dK+dV 27.6 -> 25.5 us, C5 73.8 -> 68.6); otherwise as deep as smem allows (the
    // block-sparse C4, whose column entries are mostly half empty, loses ~10 us when paired)
    static constexpr int NS_ = PAIRED ? 2 : (kSmemMax - 4096) / SB;
    static constexpr int NS = NS_ > 4 ? 4 : NS_;
    static constexpr uint32_t TMEM_COLS = 2 * D < 32 ? 32 : 2 * D;  // two D-column accumulators
    static_assert(NS >= 2, "smem budget");
    static constexpr int OFF_BAR = NS * SB;
    static constexpr int NBAR = 3 * NS + 4;
    static constexpr int OFF_OHDR = OFF_BAR + NBAR * 8;
    static constexpr int OFF_TPTR = OFF_OHDR + 2 * (int)sizeof(KHdr);
    static constexpr int SMEM = OFF_TPTR + 16 + 1024;
    static_assert(SMEM <= kSmemMax, "smem budget");
    static constexpr int THREADS = 384;
};

// One launch of 2 x n_ccta CTAs: the first n_ccta compute dV = y^T dO (PV: A = X' tiles scaled by
// r' in shared memory -> y, B = dO), the rest dK = dS'^T Q (A = dS' tiles, B = Q) for the same
// column items; dV CTAs (the heavier ones) start first, dK CTAs fill SMs as they free up.
// Warps: 0 producer, 1 MMA, 2 TMEM allocator, 4-7 y transform (PV), 8-11 epilogue.
template <int D, bool PAIRED>
__global__ void __launch_bounds__(384, 1)
    tc_bwd_kv(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmO, const Params p)
{
    const bool PV = blockIdx.x < (unsigned)p.sc.n_ccta;
    const int cta = PV ? blockIdx.x : blockIdx.x - p.sc.n_ccta;
    const CUtensorMap& tmB = PV ? tmO : tmQ;
    using C = BK<D, PAIRED>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint64_t* bars = (uint64_t*)(smem + C::OFF_BAR);
    uint64_t* full = bars;
    uint64_t* empty = full + C::NS;
    uint64_t* ready = empty + C::NS;
    uint64_t* o_full = ready + C::NS;
    uint64_t* o_empty = o_full + 2;
    KHdr* ohdr = (KHdr*)(smem + C::OFF_OHDR);
    uint32_t* tmem_ptr = (uint32_t*)(smem + C::OFF_TPTR);
    auto stage = [&](int s) { return smem + s * C::SB; };
    auto shdr = [&](int s) { return (KHdr*)(stage(s) + C::AB + C::BB + 1024); };

    const int warp = warp_uniform(), lane = threadIdx.x % 32;
    if (threadIdx.x == 0) {
        for (int i = 0; i < C::NS; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); mbar_init(&ready[i], 4); }
        for (int i = 0; i < 2; ++i) { mbar_init(&o_full[i], 2); mbar_init(&o_empty[i], 4); }
        fence_mbar_init();
    }
    if (warp == 0 && lane == 0) prefetch_tmap(&tmB);
    if (warp == 2) tmem_alloc(tmem_ptr, C::TMEM_COLS);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_ptr;
    griddep_launch_dependents();
    griddep_wait();
    const int it_begin = __ldcg(p.sc.ccta_ptr + cta), it_end = __ldcg(p.sc.ccta_ptr + cta + 1);
    const int T = p.T;
    const uint8_t* asrc = (const uint8_t*)(PV ? p.xprime : p.dsbuf);
    const int XS = kRowBlock * T * 2;

    if (warp == 0) {
        // ---------------------------------------------------------------------- producer
        const uint64_t pol_a = policy_evict_first();  // last read of dS' (dK) / X' (dV)
        int s = 0;
        uint32_t sph = 0;
        for (int it = it_begin; it < it_end; ++it) {
            const int4 d = __ldcg(p.sc.col_desc + it);
            const int g = d.x / p.sc.n_cb;
            const int64_t slot0 = (int64_t)g * p.sc.slots_per_head - d.w;
            for (int e = d.y; e < d.z; ++e) {
                const int4 ce = __ldcg(p.sc.cent + e);
                const int rb = ce.x & 0xFFFF, ha = (ce.x >> 16) & 3, hb = (ce.x >> 18) & 3;
                // key chunk ch (64 keys) comes from tile ti[ch], its 64-key column block cc[ch]
                const int ti[2] = {ce.y, T == 128 ? ce.y : ce.z};
                const int cc[2] = {0, T == 128 ? 1 : 0};
                const int hv[2] = {ce.y >= 0 ? ha : 0, T == 128 ? (ce.y >= 0 ? ha : 0) : (ce.z >= 0 ? hb : 0)};
                mbar_wait(&empty[s], sph ^ 1);
                uint8_t* st = stage(s);
                if (elect_one()) {
                    *shdr(s) = KHdr{KV_TILE, hv[0], hv[1], 0, 0, 0, 0, 0};
                    uint32_t bytes = C::AB + C::BB;
                    if (PV) bytes += (T == 128 ? 1 : (ce.y >= 0) + (ce.z >= 0)) * kRowBlock * 4;
                    mbar_arrive_expect_tx(&full[s], bytes);
                    for (int h = 0; h < D / 64; ++h)
                        tma_load_2d(st + C::AB + h * (kRowBlock * 128), &tmB, h * 64, g * p.S + rb * kRowBlock, &full[s]);
                    for (int ch = 0; ch < 2; ++ch)
                        for (int hh = 0; hh < 2; ++hh) {
                            uint8_t* dst = st + ch * (kRowBlock * 128) + hh * (kHalf * 128);
                            if (ti[ch] >= 0 && ((hv[ch] >> hh) & 1))
                                bulk_load_hint(dst, asrc + (slot0 + ti[ch]) * XS + cc[ch] * (kRowBlock * 128) + hh * (kHalf * 128),
                                               kHalf * 128, &full[s], pol_a);
                            else
                                bulk_load(dst, g_zero_half, kHalf * 128, &full[s]);
                        }
                    if (PV) {
                        uint8_t* rp = st + C::AB + C::BB;
                        if (T == 128) bulk_load(rp, p.rprime + (slot0 + ce.y) * kRowBlock, kRowBlock * 4, &full[s]);
                        else
                            for (int u = 0; u < 2; ++u)
                                if (ti[u] >= 0)
                                    bulk_load(rp + u * 512, p.rprime + (slot0 + ti[u]) * kRowBlock, kRowBlock * 4, &full[s]);
                    }
                }
                __syncwarp();
                if (++s == C::NS) { s = 0; sph ^= 1; }
            }
        }
        if (PV) {  // END for the transform warps
            mbar_wait(&empty[s], sph ^ 1);
            if (elect_one()) {
                shdr(s)->flags = KV_END;
                mbar_arrive(&full[s]);
            }
            __syncwarp();
        }
    } else if (warp == 1) {
        // ---------------------------------------------------------------------- MMA
        // D[key][d] += sum over 16-row K steps of A^T (MN-major: keys contiguous) x B (MN-major: d
        // contiguous); both operands are SW128 atoms of 8 rows x 128 B, 64-element blocks 16 KB apart
        const uint32_t idesc = idesc_f16(p.in_dtype == DT_BF16 ? 1 : 0, kRowBlock, D, 1, 1);
        int s = 0, o = 0;
        uint32_t sph = 0, oph = 0;
        auto post = [&](int flags, int64_t krow, bool second) {
            mbar_wait(&o_empty[o], oph ^ 1);
            if (elect_one()) {
                ohdr[o] = KHdr{flags, 0, 0, 0, (int32_t)(krow & 0xffffffff), (int32_t)(krow >> 32), 0, 0};
                mbar_arrive(&o_full[o]);
                if (second) mbar_arrive(&o_full[o]);
            }
            __syncwarp();
        };
        for (int it = it_begin; it < it_end; ++it) {
            const int4 d = __ldcg(p.sc.col_desc + it);
            const int g = d.x / p.sc.n_cb, c = d.x % p.sc.n_cb;
            const int64_t krow = (int64_t)g * p.S + c * kMWB;
            if (d.y == d.z) {  // no query row reaches these keys: zero gradients
                post(KV_EMPTY, krow, true);
                if (++o == 2) { o = 0; oph ^= 1; }
                continue;
            }
            post(KV_TILE, krow, false);
            const uint32_t d_tmem = tmem_base + o * D;
            for (int e = d.y; e < d.z; ++e) {
                mbar_wait(PV ? &ready[s] : &full[s], sph);
                tc_fence_after();
                const uint32_t a_addr = smem_u32(stage(s)), b_addr = a_addr + C::AB;
                if (elect_one()) {
#pragma unroll
                    for (int kk = 0; kk < kRowBlock / 16; ++kk) {
                        const uint64_t ad = smem_desc_sw128(a_addr + kk * 2048, kRowBlock * 128, 1024);
                        const uint64_t bd = smem_desc_sw128(b_addr + kk * 2048, kRowBlock * 128, 1024);
                        mma_ss(d_tmem, ad, bd, idesc, (e == d.y && kk == 0) ? 0u : 1u);
                    }
                    mma_commit(&empty[s]);
                }
                __syncwarp();
                if (++s == C::NS) { s = 0; sph ^= 1; }
            }
            if (elect_one()) mma_commit(&o_full[o]);
            __syncwarp();
            if (++o == 2) { o = 0; oph ^= 1; }
        }
        post(KV_END, 0, true);
    } else if (PV && warp >= 4 && warp < 8) {
        // ---------------------------------------------------------------------- y = X' r' in place
        const int r = (warp - 4) * 32 + lane;  // query row of the row-block
        const int myhalf = r / kHalf;
        const bool bf = p.in_dtype == DT_BF16;
        int s = 0;
        uint32_t sph = 0;
        for (;;) {
            mbar_wait(&full[s], sph);
            const KHdr h = lds_hdr(shdr(s));
            if (h.flags & KV_END) break;
            const uint32_t st = smem_u32(stage(s));
            const int hv[2] = {h.hv0, h.hv1};
#ifdef SR_DIAG_BWD_NOTRANSFORM
            if (false)
#endif
#pragma unroll
            for (int ch = 0; ch < 2; ++ch) {
                const bool valid = (hv[ch] >> myhalf) & 1;
                if (!valid) continue;  // this row of the chunk was zero-filled: y = 0 already
                const float rr = lds_f32(st + C::AB + C::BB + (T == 128 ? 0 : ch * 512) + 4 * r);
#pragma unroll
                for (int q = 0; q < 8; ++q) {
                    const uint32_t off = tile_chunk_off(r, ch * 8 + q);
                    const uint4 x = lds128(st + off);
                    const uint32_t xw[4] = {x.x, x.y, x.z, x.w};
                    uint32_t pk[4];
#pragma unroll
                    for (int w = 0; w < 4; ++w) {
                        const float2 f = unpack_f16(xw[w]);
                        pk[w] = pack16(f.x * rr, f.y * rr, bf);
                    }
                    sts128(st + off, pk[0], pk[1], pk[2], pk[3]);
                }
            }
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(&ready[s]);
            if (++s == C::NS) { s = 0; sph ^= 1; }
        }
    } else if (warp >= 8) {
        // ---------------------------------------------------------------------- epilogue
        const int r = (warp % 4) * 32 + lane;  // key of the column block == TMEM lane
        const uint32_t lane_off = (uint32_t)((warp % 4) * 32) << 16;
        void* dst = PV ? p.dv : p.dk;
        int o = 0;
        uint32_t oph = 0;
        for (;;) {
            mbar_wait(&o_full[o], oph);
            tc_fence_after();
            const KHdr h = lds_hdr(ohdr + o);
            if (h.flags & KV_END) break;
            const int64_t krow0 = ((int64_t)h.row_hi << 32) | (uint32_t)h.row_lo, krow = krow0 + r;
            const bool inhead = krow0 % p.S + r < p.S;  // S % 128 == 64: the last key block's upper half is outside
            if (h.flags & KV_EMPTY) {
                if (!inhead) {
                } else if (p.out_dtype == DT_F32) {
                    float4* O = reinterpret_cast<float4*>((float*)dst + krow * D);
                    for (int c = 0; c < D / 4; ++c) O[c] = make_float4(0.f, 0.f, 0.f, 0.f);
                } else {
                    uint4* O = reinterpret_cast<uint4*>((uint16_t*)dst + krow * D);
                    for (int c = 0; c < D / 8; ++c) O[c] = make_uint4(0, 0, 0, 0);
                }
            } else {
                const uint32_t taddr = tmem_base + lane_off + o * D;
#pragma unroll
                for (int c = 0; c < D / 32; ++c) {
                    uint32_t v[32];
                    tmem_ld32(taddr + c * 32, v);
                    tmem_wait_ld();
                    if (!inhead) {
                    } else if (p.out_dtype == DT_F32) {
                        float4* O = reinterpret_cast<float4*>((float*)dst + krow * D + c * 32);
#pragma unroll
                        for (int u = 0; u < 8; ++u)
                            O[u] = make_float4(__uint_as_float(v[4 * u]), __uint_as_float(v[4 * u + 1]),
                                               __uint_as_float(v[4 * u + 2]), __uint_as_float(v[4 * u + 3]));
                    } else {
                        uint32_t pk[16];
#pragma unroll
                        for (int u = 0; u < 16; ++u)
                            pk[u] = pack16(__uint_as_float(v[2 * u]), __uint_as_float(v[2 * u + 1]),
                                           p.out_dtype == DT_BF16);
                        uint4* O = reinterpret_cast<uint4*>((uint16_t*)dst + krow * D + c * 32);
#pragma unroll
                        for (int u = 0; u < 4; ++u) O[u] = make_uint4(pk[4 * u], pk[4 * u + 1], pk[4 * u + 2], pk[4 * u + 3]);
                    }
                }
                tc_fence_before();
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&o_empty[o]);
            if (++o == 2) { o = 0; oph ^= 1; }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, C::TMEM_COLS);
    }
}

// ------------------------------------------------------------------------------ launchers

template <int D>
cudaError_t launch_bwd_d(const Params& p, cudaStream_t st, int64_t* nl)
{
    cudaError_t e;
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    if (p.stages & 1) {
        const int64_t rpb = kPrepThreads / SR_PREP_TPR;
        if ((e = launch_pdl(bwd_prep<D>, dim3((unsigned)((rows + rpb - 1) / rpb)), dim3(kPrepThreads), 0, st, nl, p)) !=
            cudaSuccess)
            return e;
        CUtensorMap to, tv, tk;
        if ((e = make_tmap_2d(&to, p.dout, rows, D, kRowBlock, p.in_dtype)) != cudaSuccess) return e;
        if ((e = make_tmap_2d(&tv, p.v, rows, D, p.T, p.in_dtype)) != cudaSuccess) return e;
        if ((e = make_tmap_2d(&tk, p.k, rows, D, p.T, p.in_dtype)) != cudaSuccess) return e;
        auto kern = p.bwd_dq_fused ? (p.T == 64 ? tc_bwd_ds<D, 64, true> : tc_bwd_ds<D, 128, true>)
                                   : (p.T == 64 ? tc_bwd_ds<D, 64, false> : tc_bwd_ds<D, 128, false>);
        const int smem = p.bwd_dq_fused ? BD<D, true>::SMEM : BD<D, false>::SMEM;
        if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess)
            return e;
        if ((e = launch_pdl(kern, dim3(p.sc.n_cta), dim3(BD<D>::THREADS), smem, st, nl, to, tv, tk, p)) != cudaSuccess)
            return e;
    }
    if ((p.stages & 2) && !p.bwd_dq_fused) {  // dQ = dS' K: GEMM2 in its plain mode, A = dS' tiles, B = K
        Params p2 = p;
        p2.pbuf = p.dsbuf;
        p2.v = p.k;
        p2.out = p.dq;
        if ((e = launch_gemm2(p2, 0, st, nl)) != cudaSuccess) return e;
    }
    if (p.stages & 4) {
        CUtensorMap tq, to;
        if ((e = make_tmap_2d(&tq, p.q, rows, D, kRowBlock, p.in_dtype)) != cudaSuccess) return e;
        if ((e = make_tmap_2d(&to, p.dout, rows, D, kRowBlock, p.in_dtype)) != cudaSuccess) return e;
        const bool paired = D == 64 && p.mask_kind != MK_BLOCK;
        auto kern = paired ? tc_bwd_kv<D, D == 64> : tc_bwd_kv<D, false>;
        const int ksmem = paired ? BK<D, D == 64>::SMEM : BK<D, false>::SMEM;
        if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, ksmem)) != cudaSuccess)
            return e;
        if ((e = launch_pdl(kern, dim3(2 * p.sc.n_ccta), dim3(BK<D>::THREADS), ksmem, st, nl, tq, to, p)) !=
            cudaSuccess)
            return e;
    }
    return cudaSuccess;
}

cudaError_t launch_tc_bwd(const Params& p, cudaStream_t st, int64_t* nl)
{
    return p.D == 64 ? launch_bwd_d<64>(p, st, nl) : launch_bwd_d<128>(p, st, nl);
}

}  // namespace sr
