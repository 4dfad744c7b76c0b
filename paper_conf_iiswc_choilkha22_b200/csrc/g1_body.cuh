// g1_body.cuh -- GEMM1 (device code shared by tc_gemm1 in k_g1.cu and the fused kernel in k_fused.cu) = Q K^T with scale + mask, and the Local Softmax (LS) sub-layer fused into
// its epilogue ("setting T of the LS kernel equal to the output tile width
// of the MatMul kernel, the LS kernel can be fused to its preceding MatMul kernel"; scale and mask
// fused as element-wise layers, L169).  LS=false builds the unfused baseline's GEMM1, which writes
// the scaled, masked score tile S instead (L171).
//
// Per 128-row x T-key sub-tile (the LS sub-vector, T = 64 or 128), fp32 accumulator in TMEM:
//   m'  = max_j x_j                    (x = Q K^T * scale, masked to -inf)
//   X'  = e^{x - m'}  -> fp16 tile, written to HBM once (the only attention-matrix write)
//   d'  = sum_j X'_j                   (fp32)
// m', d' go to the workspace as fp32 [slot][128 rows].
//
// Macro tiles.  The tensor core always computes 128 x MW (MW = 128) score tiles: with T = 64 two
// consecutive sub-tiles of the item's key list (any two key blocks, stacked in one K stage) share
// one N = 128 MMA, each keeping its own mask, statistics, validity and slot (consecutive list
// entries are adjacent slots, so the pair's X' is contiguous in HBM).
//
// Warp roles (persistent CTA per SM, 640 threads for T = 64, 384 for T = 128):
//   warp 0      TMA producer: Q tile per item, K blocks of each macro tile (NK-stage ring)
//   warp 1      MMA issuer: D/16 tcgen05.mma kind::f16 of 128 x MW x 16 per macro tile into one of
//               NACC TMEM accumulators; publishes a header (slot, rows, key tiles, half-valid bits,
//               kv_len) next to the accumulator -- acc_full completes when both the header arrive and
//               the MMA commit have landed
//   warp 2      TMEM allocator (512 columns)
//   epilogue    T = 64 (SPLIT): warps 4-19, four warpgroups; a pair takes every other macro tile,
//               one warpgroup per 64-key sub-tile.  T = 128 (FULL): warps 4-11, two warpgroups taking
//               alternate macro tiles, full 128-key rows.  Each warp: one tcgen05.ld of its row's
//               scores, accumulator released at once, interval-bitmask mask, max, FFMA2 + ex2, FADD2
//               sums, fp16 pack, st.shared into a swizzled staging tile, a bulk store of its own rows.
//               (Splitting a T = 128 row across warpgroups needs a max/sum exchange that costs more
//               than it saves -- measured.)
#pragma once
#include "tc_common.cuh"

namespace sr {

using namespace ptx;

#ifdef SR_DIAG_WAITS
static __device__ unsigned long long g_diag_g1[32 * (kDW + 1)];
#endif

constexpr int kMW = 128;  // macro tile width (MMA N of GEMM1)
#ifndef SR_G1_QPREFETCH
#define SR_G1_QPREFETCH 0
#endif
constexpr bool kQPrefetch = SR_G1_QPREFETCH;  // L2 prefetch of the next item's Q (measured: C3 slower, off)
#ifndef SR_G1_HINTS
#define SR_G1_HINTS 1
#endif
#ifndef SR_G1_KHINT
#define SR_G1_KHINT SR_G1_HINTS
#endif
constexpr bool kG1KHint = SR_G1_KHINT;  // K loads evict_last (re-read by every row-block)
// X' stores: evict_first (streamed) only when the layer's X' does not fit comfortably in L2
// (p.x_evict_first, chosen on the host); a small X' stays at normal priority and is read back from L2
// Of every 8 element pairs of the LS exponentials, this many are computed by ex2_poly2 on the FMA
// pipe and the rest by MUFU.EX2 (16 / clock / SM): balances the two pipes in the epilogue.
#ifndef SR_G1_POLY_PAIRS
#define SR_G1_POLY_PAIRS 0
#endif
constexpr int kPolyPairs = SR_G1_POLY_PAIRS;

struct G1Hdr {  // per-accumulator macro-tile header, written by the MMA warp
    int32_t slot_lo, slot_hi, i0, kvl, w0, w1, flags, pad;
};
// HDR_LASTT / HDR_MARK (concurrent kernel): the header ends item (flags >> 8) of the CTA's list --
// its last tile, or a tile-less notice to the other epilogue warpgroup (both for an empty item)
enum : int { HDR_TILE = 1, HDR_END = 2, HDR_KEEP = 4, HDR_LASTT = 8, HDR_MARK = 16 };

template <int D, int T, bool PAIR, int MW_ = kMW, int BUDGET = kSmemMax>
struct G1 {
    // MW_ = 64 / BUDGET < kSmemMax: the concurrent kernel's GEMM1 half (k_conc.cu): 64-key macro
    // tiles, two 64-column TMEM accumulators, FULL epilogue (one warpgroup per macro tile)
    static constexpr int MW = MW_;                // macro tile width (MMA N)
    static constexpr int NSUB = MW / T;           // sub-tiles per macro tile
    static constexpr int QB = kRowBlock * D * 2;  // Q tile bytes
    static constexpr int QS = (PAIR ? 2 : 1) * QB;  // Q stage: one row-block, or a pair
    static constexpr int KB = MW * D * 2;         // K stage bytes (MW keys)
    static constexpr bool SPLIT = (T == 64 && MW == 128);  // epilogue organisation, see the file header
    static constexpr int EPI_WG = SPLIT ? 4 : 2;  // epilogue warpgroups
    static constexpr int HB = kRowBlock * 64 * 2;  // SPLIT staging tile: one warpgroup's 64 columns
    static constexpr int XB2 = kRowBlock * MW * 2;  // FULL staging tile: a whole macro tile
    static constexpr int SB = SPLIT ? HB : XB2;    // staging buffer per warpgroup
    static constexpr int XS = kRowBlock * T * 2;  // X' slot bytes (sub-tile)
    static constexpr int NACC = MW == 128 ? 4 : 2;  // TMEM accumulators (512 or 128 columns)
    // staging buffers per epilogue warpgroup (2 if at all possible: the X' store stream is the
    // bottleneck), then Q double-buffered if shared memory still allows
    // statistics ring for the IR-in-GEMM1 variant: per accumulator, NSUB x (m', d') x 128 rows fp32
    static constexpr int STB = NACC * 2 * 2 * kRowBlock * 4;
    static constexpr int SLACK = (BUDGET == kSmemMax ? 4096 : 1024) + STB;
    static constexpr int XPW = ((PAIR ? 2 * QS : QS) + 2 * KB + EPI_WG * 2 * SB + SLACK <= BUDGET) ? 2 : 1;
#ifndef SR_G1_MAX_NQ
#define SR_G1_MAX_NQ 2
#endif
    static constexpr int NQ = (SR_G1_MAX_NQ >= 2 && 2 * QS + 2 * KB + EPI_WG * XPW * SB + SLACK <= BUDGET) ? 2 : 1;
    static constexpr int NK_ = (BUDGET - SLACK - NQ * QS - EPI_WG * XPW * SB) / KB;
    static constexpr int NK_MAX = MW == 128 ? 4 : 6;
    static constexpr int NK = NK_ > NK_MAX ? NK_MAX : NK_;
    static_assert(NK >= 2, "smem budget");
    static constexpr int OFF_Q = 0;
    static constexpr int OFF_K = OFF_Q + NQ * QS;
    static constexpr int OFF_X = OFF_K + NK * KB;
    static constexpr int OFF_BAR = OFF_X + EPI_WG * XPW * SB;
    static constexpr int NBAR = 2 * NQ + 2 * NK + 4 * NACC;
    static constexpr int OFF_STATS = OFF_BAR + NBAR * 8;
    static constexpr int OFF_HDR = OFF_STATS + STB;
    static constexpr int OFF_TPTR = OFF_HDR + NACC * (int)sizeof(G1Hdr);
    static constexpr int SMEM_ = OFF_TPTR + 16 + 1024;  // + alignment slack
    static constexpr int SMEM = (BUDGET == kSmemMax && SMEM_ < 118 * 1024) ? 118 * 1024 : SMEM_;  // 1 CTA/SM
    static_assert(SMEM <= kSmemMax, "smem budget");
    static constexpr int THREADS = 128 + EPI_WG * 128;
};

// IRT: the IR sub-layer runs in this kernel (the default mode): every CTA owns whole rows (all key
// tiles of its row-blocks), so warp 3 merges the epilogue's per-tile (m', d') of each row as they
// are produced and, at the end of the row-block, writes the row's (m, 1/d) -- see the IR warp below.
// Barrier initialisation of GEMM1's shared-memory layout (thread 0; fence_mbar_init included).
template <int D, int T, bool LS, bool PAIR, bool IRT, int MW = kMW, int BUDGET = kSmemMax>
__device__ __forceinline__ void g1_init(uint8_t* smem)
{
    using C = G1<D, T, PAIR, MW, BUDGET>;
    constexpr bool SPLIT = C::SPLIT;
    uint64_t* bars = (uint64_t*)(smem + C::OFF_BAR);
    uint64_t* q_full = bars;
    uint64_t* q_empty = q_full + C::NQ;
    uint64_t* k_full = q_empty + C::NQ;
    uint64_t* k_empty = k_full + C::NK;
    uint64_t* acc_full = k_empty + C::NK;
    uint64_t* acc_empty = acc_full + C::NACC;
    uint64_t* st_full = acc_empty + C::NACC;
    uint64_t* st_empty = st_full + C::NACC;
    if (threadIdx.x == 0) {
        for (int i = 0; i < C::NQ; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
        for (int i = 0; i < C::NK; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
        // acc_full: header arrive (MMA thread) + tcgen05.commit; acc_empty: one arrive per epilogue
        // warp that reads the accumulator (the warpgroup pair in SPLIT, one warpgroup in FULL)
        for (int i = 0; i < C::NACC; ++i) { mbar_init(&acc_full[i], 2); mbar_init(&acc_empty[i], SPLIT ? 8 : 4); }
        for (int i = 0; i < C::NACC; ++i) { mbar_init(&st_full[i], SPLIT ? 8 : 4); mbar_init(&st_empty[i], 1); }
        fence_mbar_init();
    }
}

// Warp roles of GEMM1 (everything after the prologue): TMA producer, MMA issuer, IR warps,
// epilogue warpgroups; uses every warp of the CTA (384 threads for T = 128, 640 for T = 64).
// CONC (concurrent kernel, k_conc.cu): GEMM2 runs beside this GEMM1 in the same CTA and takes each
// item over as soon as it is complete.  `ibar` = item_done[kConcNI] (10 arrivals per item: the eight
// epilogue warps once their X' stores and m' of the item have landed, the two IR warps once its
// row statistics are written) followed by item_free[kConcNI] (GEMM2 has taken the item; the MMA warp
// waits on it before starting the item kConcNI places later).
template <int D, int T, bool LS, bool PAIR, bool IRT, bool REGS = true, int MW = kMW, int BUDGET = kSmemMax,
          bool CONC = false, int RM = 3>
__device__ __forceinline__ void g1_roles(const CUtensorMap& tmQ, const CUtensorMap& tmK, const Params& p,
                                          const DevSched& sc, uint8_t* smem, uint32_t tmem_base, int it_begin,
                                          int it_end, uint64_t* ibar = nullptr)
{
    using C = G1<D, T, PAIR, MW, BUDGET>;
    static_assert(!CONC || (!PAIR && !C::SPLIT && IRT), "concurrent kernel: unpaired FULL epilogue, IR in GEMM1");
    uint64_t* item_done = ibar;
    uint64_t* item_free = CONC ? ibar + kConcNI : nullptr;
    constexpr int NSUB = C::NSUB;
    constexpr bool SPLIT = C::SPLIT;
    uint64_t* bars = (uint64_t*)(smem + C::OFF_BAR);
    uint64_t* q_full = bars;
    uint64_t* q_empty = q_full + C::NQ;
    uint64_t* k_full = q_empty + C::NQ;
    uint64_t* k_empty = k_full + C::NK;
    uint64_t* acc_full = k_empty + C::NK;
    uint64_t* acc_empty = acc_full + C::NACC;
    uint64_t* st_full = acc_empty + C::NACC;  // IRT: per-accumulator (m', d') of its rows staged
    uint64_t* st_empty = st_full + C::NACC;   // IRT: ... and merged by the IR warp
    float* stats = (float*)(smem + C::OFF_STATS);  // [NACC][NSUB][m' | d'][128]
    G1Hdr* hdr = (G1Hdr*)(smem + C::OFF_HDR);
    uint32_t* tmem_ptr = (uint32_t*)(smem + C::OFF_TPTR);

    const int warp = warp_uniform(), lane = threadIdx.x % 32;
    DW_DECL
    const uint64_t pol_k = kG1KHint ? policy_evict_last() : 0, pol_x = p.x_evict_first ? policy_evict_first() : 0;
    auto kload = [&](void* d, const CUtensorMap* m, int c0, int c1, uint64_t* b) {
        if (kG1KHint) tma_load_2d_hint(d, m, c0, c1, b, pol_k);
        else tma_load_2d(d, m, c0, c1, b);
    };
    // the CTA's items in processing order: last-first with p.p1_reverse (LPT order is longest first,
    // so the largest items are then processed -- and their X' written -- last, see k_fused.cu)
    auto p1at = [&](int j) { return p.p1_reverse ? it_begin + it_end - 1 - j : j; };
    auto xstore = [&](void* d, const void* src, uint32_t nb, bool keep) {
        if (p.x_evict_first && !keep) bulk_store_hint(d, src, nb, pol_x);
        else bulk_store(d, src, nb);
    };

    // RM: role groups compiled into this call (1: warps 0-3, 2: epilogue warpgroups), so a caller can
    // run each group under its own setmaxnreg budget (k_conc.cu)
    if ((RM & 1) && (!(RM & 2) || warp < 4)) {
        // warpgroup 0 hands registers to the epilogue warpgroups.  setmaxnreg.inc can only draw what
        // other warps of this CTA released, so the budgets balance exactly:
        //   SPLIT (640 threads, 96 at launch): 4 warps x 32 x (96 - 64) = 16 warps x 32 x (104 - 96)
        //   FULL  (384 threads, 168 at launch): 4 warps x 32 x (168 - 56) = 8 warps x 32 x (224 - 168)
        if constexpr (!REGS) {  // no rebalancing (the fused kernel's chunk loop: see k_fused.cu)
        } else if constexpr (SPLIT) reg_dealloc<64>();
        else reg_dealloc<56>();
        if (PAIR && warp == 0) {
            // -------------------------------------------------------------- TMA producer, pairs:
            // Q of row-blocks 2j and 2j+1 per item, then one K stage per union macro tile
            int qi = 0, ks = 0;
            uint32_t qph = 0, kph = 0;
            int4 nd = it_begin < it_end ? __ldca(sc.pair_desc + p1at(it_begin)) : make_int4(0, 0, 0, 0);
            for (int it = it_begin; it < it_end; ++it) {
                const int4 d = nd;
                if (it + 1 < it_end) nd = __ldca(sc.pair_desc + p1at(it + 1));
                const int g = d.x / sc.n_pair, j = d.x % sc.n_pair, e0 = d.y, e1 = d.z;
                if (e0 == e1) continue;
                const int nrb = 2 * j + 1 < sc.n_rb ? 2 : 1;
                const int row0 = g * p.S + 2 * j * kRowBlock;
                DW_WAIT(&q_empty[qi], qph ^ 1, 0);
                if (elect_one()) {
                    mbar_arrive_expect_tx(&q_full[qi], nrb * C::QB);
                    for (int r = 0; r < nrb; ++r)
                        for (int h = 0; h < D / 64; ++h)
                            tma_load_2d(smem + C::OFF_Q + qi * C::QS + r * C::QB + h * (kRowBlock * 128), &tmQ, h * 64,
                                        row0 + r * kRowBlock, &q_full[qi]);
                    if (kQPrefetch && it + 1 < it_end) {  // the next item's Q into L2 (Q is single-buffered)
                        const int g2 = nd.x / sc.n_pair, j2 = nd.x % sc.n_pair;
                        const int nrb2 = 2 * j2 + 1 < sc.n_rb ? 2 : 1;
                        for (int r = 0; r < nrb2; ++r)
                            for (int h = 0; h < D / 64; ++h)
                                tma_prefetch_2d(&tmQ, h * 64, g2 * p.S + (2 * j2 + r) * kRowBlock);
                    }
                }
                __syncwarp();
                if (++qi == C::NQ) { qi = 0; qph ^= 1; }
                int wn[NSUB];
#pragma unroll
                for (int s2 = 0; s2 < NSUB; ++s2) wn[s2] = e0 + s2 < e1 ? __ldca(&sc.pent[e0 + s2].x) : 0;
                for (int e = e0; e < e1; e += NSUB) {
                    const int nsub = min(NSUB, e1 - e);
                    int w[NSUB];
#pragma unroll
                    for (int s2 = 0; s2 < NSUB; ++s2) {
                        w[s2] = wn[s2];
                        wn[s2] = e + NSUB + s2 < e1 ? __ldca(&sc.pent[e + NSUB + s2].x) : 0;
                    }
                    DW_WAIT(&k_empty[ks], kph ^ 1, 1);
                    if (elect_one()) {
                        mbar_arrive_expect_tx(&k_full[ks], nsub * T * D * 2);
                        for (int s2 = 0; s2 < nsub; ++s2)
                            for (int h = 0; h < D / 64; ++h)
                                kload(smem + C::OFF_K + ks * C::KB + h * (C::MW * 128) + s2 * (T * 128), &tmK,
                                            h * 64, g * p.S + (w[s2] & 0xFFFF) * T, &k_full[ks]);
                    }
                    __syncwarp();
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                }
            }
        } else if (PAIR && warp == 1) {
            // -------------------------------------------------------------- MMA issuer, pairs: per
            // union macro tile, the MMAs of each row-block that has a valid sub-tile in it, each into
            // the next TMEM accumulator of the common ring (the epilogue is the same as unpaired)
            const uint32_t idesc = idesc_f16(p.in_dtype == DT_BF16 ? 1 : 0, kRowBlock, C::MW, 0, 0);
            int qi = 0, ks = 0, n = 0;
            uint32_t qph = 0, kph = 0;
            int4 nd = it_begin < it_end ? __ldca(sc.pair_desc + p1at(it_begin)) : make_int4(0, 0, 0, 0);
            for (int it = it_begin; it < it_end; ++it) {
                const int4 d = nd;
                if (it + 1 < it_end) nd = __ldca(sc.pair_desc + p1at(it + 1));
                const int g = d.x / sc.n_pair, j = d.x % sc.n_pair, e0 = d.y, e1 = d.z;
                if (e0 == e1) continue;
                const int nrb = 2 * j + 1 < sc.n_rb ? 2 : 1;
                const int kvl = sc.kv_len ? __ldca(sc.kv_len + g / p.H) : p.S;
                const int64_t slot0 = (int64_t)g * sc.slots_per_head - d.w;
                DW_WAIT(&q_full[qi], qph, 0);
                tc_fence_after();
                const uint32_t q_addr = smem_u32(smem + C::OFF_Q + qi * C::QS);
                int4 wn[NSUB];
#pragma unroll
                for (int s2 = 0; s2 < NSUB; ++s2) wn[s2] = e0 + s2 < e1 ? __ldca(sc.pent + e0 + s2) : make_int4(0, -1, -1, 0);
                for (int e = e0; e < e1; e += NSUB) {
                    int4 w[NSUB];
#pragma unroll
                    for (int s2 = 0; s2 < NSUB; ++s2) {
                        w[s2] = wn[s2];
                        wn[s2] = e + NSUB + s2 < e1 ? __ldca(sc.pent + e + NSUB + s2) : make_int4(0, -1, -1, 0);
                    }
                    DW_WAIT(&k_full[ks], kph, 1);
                    tc_fence_after();
                    const uint32_t k_addr = smem_u32(smem + C::OFF_K + ks * C::KB);
                    for (int r = 0; r < nrb; ++r) {
                        int ws[2] = {-1, -1};
                        int64_t sl[2] = {0, 0};
#pragma unroll
                        for (int s2 = 0; s2 < NSUB; ++s2) {
                            const int hb = (w[s2].x >> (16 + 2 * r)) & 3;
                            if (e + s2 < e1 && hb) {
                                ws[s2] = (w[s2].x & 0xFFFF) | (hb << 16);
                                sl[s2] = slot0 + (r ? w[s2].z : w[s2].y);
                            }
                        }
                        if (ws[0] == -1 && ws[1] == -1) continue;  // nothing of this row-block here
                        const int buf = n % C::NACC;
                        DW_WAIT(&acc_empty[buf], ((n / C::NACC) & 1) ^ 1, 2);
                        // sub-tile s's slot = slot + (s ? dslot : 0)
                        const int64_t slot = ws[0] != -1 ? sl[0] : sl[1];
                        const int dslot = (ws[0] != -1 && ws[1] != -1) ? (int)(sl[1] - sl[0]) : 0;
                        if (elect_one()) {
                            hdr[buf] = G1Hdr{(int32_t)(slot & 0xffffffff), (int32_t)(slot >> 32),
                                             (2 * j + r) * kRowBlock, kvl, ws[0], ws[1],
                                             HDR_TILE | (it >= it_end - p.x_keep ? HDR_KEEP : 0), dslot};
                            mbar_arrive(&acc_full[buf]);  // header published (arrival 1 of 2)
                        }
                        __syncwarp();
                        const uint32_t d_tmem = tmem_base + buf * C::MW;
                        const uint32_t qa = q_addr + r * C::QB;
                        if (elect_one()) {
#pragma unroll
                            for (int kk = 0; kk < D / 16; ++kk) {
                                const uint32_t h = kk / 4, wk = kk % 4;
                                const uint64_t ad = smem_desc_sw128(qa + h * (kRowBlock * 128) + wk * 32, 16, 1024);
                                const uint64_t bd = smem_desc_sw128(k_addr + h * (C::MW * 128) + wk * 32, 16, 1024);
                                mma_ss(d_tmem, ad, bd, idesc, kk > 0 ? 1u : 0u);
                            }
                            mma_commit(&acc_full[buf]);  // arrival 2 of 2 when the MMAs complete
                        }
                        __syncwarp();
                        ++n;
                    }
                    if (elect_one()) mma_commit(&k_empty[ks]);
                    __syncwarp();
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                }
                if (elect_one()) mma_commit(&q_empty[qi]);
                __syncwarp();
                if (++qi == C::NQ) { qi = 0; qph ^= 1; }
            }
            for (int e = 0; e < 2; ++e, ++n) {  // one END header for each epilogue warpgroup (pair)
                const int buf = n % C::NACC;
                DW_WAIT(&acc_empty[buf], ((n / C::NACC) & 1) ^ 1, 2);
                if (elect_one()) {
                    hdr[buf].flags = HDR_END;
                    mbar_arrive(&acc_full[buf]);
                    mbar_arrive(&acc_full[buf]);
                }
                __syncwarp();
            }
        } else if (warp == 0) {
            // -------------------------------------------------------------- TMA producer (whole
            // warp walks the schedule; one elected lane issues)
            int qi = 0, ks = 0;
            uint32_t qph = 0, kph = 0;
            for (ItemWalk iw(sc, it_begin, it_end, p.p1_reverse); iw.more();) {
                const ItemInfo I = iw.next();
                if (I.t0 == I.t1) continue;
                const int row0 = I.g * p.S + I.rb * kRowBlock;
                DW_WAIT(&q_empty[qi], qph ^ 1, 0);
                if (elect_one()) {
                    mbar_arrive_expect_tx(&q_full[qi], C::QB);
                    for (int h = 0; h < D / 64; ++h)
                        tma_load_2d(smem + C::OFF_Q + qi * C::QB + h * (kRowBlock * 128), &tmQ, h * 64, row0, &q_full[qi]);
                }
                __syncwarp();
                if (++qi == C::NQ) { qi = 0; qph ^= 1; }
                int wn[NSUB];  // schedule words of the next macro tile, prefetched one step ahead
#pragma unroll
                for (int s = 0; s < NSUB; ++s) wn[s] = I.t0 + s < I.t1 ? __ldca(sc.tinfo + I.t0 + s) : 0;
                for (int t = I.t0; t < I.t1; t += NSUB) {
                    const int nsub = min(NSUB, I.t1 - t);
                    int w[NSUB];
#pragma unroll
                    for (int s = 0; s < NSUB; ++s) {
                        w[s] = wn[s];
                        wn[s] = t + NSUB + s < I.t1 ? __ldca(sc.tinfo + t + NSUB + s) : 0;
                    }
                    DW_WAIT(&k_empty[ks], kph ^ 1, 1);
                    if (elect_one()) {
#ifdef SR_DIAG_NOKLOAD
                        mbar_arrive(&k_full[ks]);
                        if (false)
#else
                        mbar_arrive_expect_tx(&k_full[ks], nsub * T * D * 2);
#endif
                        for (int s = 0; s < nsub; ++s)
                            for (int h = 0; h < D / 64; ++h)
                                kload(smem + C::OFF_K + ks * C::KB + h * (C::MW * 128) + s * (T * 128), &tmK,
                                            h * 64, I.g * p.S + tinfo_kt(w[s]) * T, &k_full[ks]);
                    }
                    __syncwarp();
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                }
            }
        } else if (warp == 1) {
            // -------------------------------------------------------------- MMA issuer (whole warp
            // walks the schedule; one elected lane issues)
            const uint32_t idesc = idesc_f16(p.in_dtype == DT_BF16 ? 1 : 0, kRowBlock, C::MW, 0, 0);
            int qi = 0, ks = 0, n = 0;
            uint32_t qph = 0, kph = 0;
            // CONC: item-end notices for the epilogue warpgroup(s) that did not get the item's last
            // tile (tile-less headers: no MMA, both acc_full arrivals from here)
            auto post_marks = [&](int cnt, int kord) {
                for (int e = 0; e < cnt; ++e, ++n) {
                    const int ab = n % C::NACC;
                    DW_WAIT(&acc_empty[ab], ((n / C::NACC) & 1) ^ 1, 2);
                    if (elect_one()) {
                        hdr[ab].flags = HDR_MARK | (kord << 8);
                        mbar_arrive(&acc_full[ab]);
                        mbar_arrive(&acc_full[ab]);
                    }
                    __syncwarp();
                }
            };
            for (ItemWalk iw(sc, it_begin, it_end, p.p1_reverse); iw.more();) {
                const bool keep = iw.it >= it_end - p.x_keep;  // before next(): the index of this item
                const int kord = iw.it - it_begin;             // CONC: the item's place in the CTA's list
                const ItemInfo I = iw.next();
                // CONC: at most kConcNI items ahead of GEMM2 (bounds the X' in flight, keeps it in L2)
                if constexpr (CONC) DW_WAIT(&item_free[kord % kConcNI], ((kord / kConcNI) & 1) ^ 1, 3);
                if (I.t0 == I.t1) {
                    if constexpr (CONC) post_marks(2, kord);
                    continue;
                }
                const int kvl = sc.kv_len ? __ldca(sc.kv_len + I.g / p.H) : p.S;
                DW_WAIT(&q_full[qi], qph, 0);
                tc_fence_after();
                const uint32_t q_addr = smem_u32(smem + C::OFF_Q + qi * C::QB);
                int wn0 = __ldca(sc.tinfo + I.t0), wn1 = (NSUB > 1 && I.t0 + 1 < I.t1) ? __ldca(sc.tinfo + I.t0 + 1) : -1;
                for (int t = I.t0; t < I.t1; t += NSUB, ++n) {
                    const int w0 = wn0, w1 = NSUB > 1 ? wn1 : -1;
                    if (t + NSUB < I.t1) wn0 = __ldca(sc.tinfo + t + NSUB);  // prefetch the next macro tile
                    wn1 = (NSUB > 1 && t + NSUB + 1 < I.t1) ? __ldca(sc.tinfo + t + NSUB + 1) : -1;
                    const int ab = n % C::NACC;
                    DW_WAIT(&acc_empty[ab], ((n / C::NACC) & 1) ^ 1, 2);
                    const int64_t slot = I.slot0 + t;
                    if (elect_one()) {
                        const int last = (CONC && t + NSUB >= I.t1) ? (HDR_LASTT | (kord << 8)) : 0;
                        hdr[ab] = G1Hdr{(int32_t)(slot & 0xffffffff), (int32_t)(slot >> 32), I.rb * kRowBlock, kvl, w0,
                                        w1, HDR_TILE | (keep ? HDR_KEEP : 0) | last, 1};  // adjacent sub-tile slots
                        mbar_arrive(&acc_full[ab]);  // header published (arrival 1 of 2)
                    }
                    __syncwarp();
                    DW_WAIT(&k_full[ks], kph, 1);
                    tc_fence_after();
                    const uint32_t k_addr = smem_u32(smem + C::OFF_K + ks * C::KB);
                    const uint32_t d_tmem = tmem_base + ab * C::MW;
                    if (elect_one()) {
#pragma unroll
                        for (int kk = 0; kk < D / 16; ++kk) {
                            const uint32_t h = kk / 4, wk = kk % 4;
                            const uint64_t ad = smem_desc_sw128(q_addr + h * (kRowBlock * 128) + wk * 32, 16, 1024);
                            const uint64_t bd = smem_desc_sw128(k_addr + h * (C::MW * 128) + wk * 32, 16, 1024);
                            mma_ss(d_tmem, ad, bd, idesc, kk > 0 ? 1u : 0u);
                        }
                        mma_commit(&k_empty[ks]);
                        mma_commit(&acc_full[ab]);  // arrival 2 of 2 when the MMAs complete
                    }
                    __syncwarp();
                    if (++ks == C::NK) { ks = 0; kph ^= 1; }
                }
                if (elect_one()) mma_commit(&q_empty[qi]);
                __syncwarp();
                if (++qi == C::NQ) { qi = 0; qph ^= 1; }
                if constexpr (CONC) post_marks(1, kord);
            }
            for (int e = 0; e < 2; ++e, ++n) {  // one END header for each epilogue warpgroup pair
                const int ab = n % C::NACC;
                DW_WAIT(&acc_empty[ab], ((n / C::NACC) & 1) ^ 1, 2);
                if (elect_one()) {
                    hdr[ab].flags = HDR_END;
                    mbar_arrive(&acc_full[ab]);
                    mbar_arrive(&acc_full[ab]);
                }
                __syncwarp();
            }
        } else if (IRT && (warp == 2 || warp == 3)) {
            // -------------------------------------------------------------- IR warps (default mode)
            // The IR sub-layer of every row this CTA owns: merge the staged
            // (m'_k, d'_k) of each row into a running
            //   m = max_k m'_k,   d = sum_k e^{m'_k - m} d'_k
            // Warp 2 takes the even accumulators (epilogue warpgroup / pair 0), warp 3 the odd ones,
            // so the two epilogue streams never wait on each other through the statistics ring; at a
            // row-block's end each warp writes its partial (m_w in natural-log units, d_w) to its
            // half of `rowstat`, and GEMM2 merges the two partials into the row's (m, 1/d) and forms
            // r'_k = e^{m'_k - m} / d in its prologue.  Lane l owns rows l + 32 j of a row-block.
            const float sl2 = p.scale_log2;
            const int par = warp - 2;
            int n = 0;
            auto merge = [&](float (&m)[4], float (&d)[4]) {
#ifdef SR_DIAG_NOSTATS
                if (false) {
#else
                if ((n & 1) == par) {
#endif
                    const int buf = n % C::NACC;
                    DW_WAIT(&st_full[buf], (uint32_t)(n / C::NACC) & 1, 0);
                    const float* sb = stats + buf * (4 * kRowBlock) + lane;
                    float mk[4][NSUB], dk[4][NSUB];
#pragma unroll
                    for (int j = 0; j < 4; ++j)
#pragma unroll
                        for (int s = 0; s < NSUB; ++s) {
                            mk[j][s] = sb[(2 * s) * kRowBlock + 32 * j];  // raw score units, -inf if invalid
                            dk[j][s] = sb[(2 * s + 1) * kRowBlock + 32 * j];
                        }
                    __syncwarp();  // every lane's reads of the stage are done
                    if (lane == 0) mbar_arrive(&st_empty[buf]);
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        float mn = m[j];
#pragma unroll
                        for (int s = 0; s < NSUB; ++s) mn = fmaxf(mn, mk[j][s]);
                        if (mn != -INFINITY) {  // ex2(-inf) = 0 covers empty sides
                            float acc = d[j] * ex2((m[j] - mn) * sl2);
#pragma unroll
                            for (int s = 0; s < NSUB; ++s) acc = fmaf(dk[j][s], ex2((mk[j][s] - mn) * sl2), acc);
                            d[j] = acc;
                            m[j] = mn;
                        }
                    }
                }
                ++n;
            };
            // CONC: an item-end notice occupies a slot of the statistics ring without data
            auto skip_mark = [&]() {
                if ((n & 1) == par) {
                    const int buf = n % C::NACC;
                    DW_WAIT(&st_full[buf], (uint32_t)(n / C::NACC) & 1, 0);
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&st_empty[buf]);
                }
                ++n;
            };
            auto flush = [&](int g, int rb, const float (&m)[4], const float (&d)[4]) {
                const int64_t nrow = (int64_t)p.B * p.H * p.Spad;  // rowstat rows: per head, whole row-blocks
                const int64_t row = (int64_t)g * p.Spad + rb * kRowBlock + lane + 2 * par * nrow;
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    p.rowstat[row + 32 * j] = m[j] * p.scale;  // -inf stays -inf
                    p.rowstat[nrow + row + 32 * j] = d[j];
                }
            };
            if (PAIR) {
                int4 nd = it_begin < it_end ? __ldca(sc.pair_desc + p1at(it_begin)) : make_int4(0, 0, 0, 0);
                for (int it = it_begin; it < it_end; ++it) {
                    const int4 dd = nd;
                    if (it + 1 < it_end) nd = __ldca(sc.pair_desc + p1at(it + 1));
                    const int g = dd.x / sc.n_pair, j = dd.x % sc.n_pair, e0 = dd.y, e1 = dd.z;
                    if (e0 == e1) continue;
                    const int nrb = 2 * j + 1 < sc.n_rb ? 2 : 1;
                    float m0[4], d0[4], m1[4], d1[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) { m0[u] = m1[u] = -INFINITY; d0[u] = d1[u] = 0.f; }
                    for (int e = e0; e < e1; e += NSUB) {
                        int hb = 0;  // union of the sub-tiles' half bits: bits 0-1 row-block 0, 2-3 row-block 1
#pragma unroll
                        for (int s2 = 0; s2 < NSUB; ++s2)
                            if (e + s2 < e1) hb |= (__ldca(&sc.pent[e + s2].x) >> 16) & 15;
                        if (hb & 3) merge(m0, d0);
                        if (nrb == 2 && (hb & 12)) merge(m1, d1);
                    }
                    flush(g, 2 * j, m0, d0);
                    if (nrb == 2) flush(g, 2 * j + 1, m1, d1);
                }
            } else {
                for (ItemWalk iw(sc, it_begin, it_end, p.p1_reverse); iw.more();) {
                    const int kord = iw.it - it_begin;
                    const ItemInfo I = iw.next();
                    if (I.t0 == I.t1) {
                        if constexpr (CONC) {  // the item's two tile-less notices; nothing to merge
                            skip_mark();
                            skip_mark();
                            if (lane == 0) mbar_arrive(&item_done[kord % kConcNI]);
                        }
                        continue;
                    }
                    float m[4], d[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) { m[u] = -INFINITY; d[u] = 0.f; }
                    for (int t = I.t0; t < I.t1; t += NSUB) merge(m, d);
                    flush(I.g, I.rb, m, d);
                    if constexpr (CONC) {  // the item-end notice; rowstat of the item is written
                        skip_mark();
                        __syncwarp();
                        if (lane == 0) mbar_arrive(&item_done[kord % kConcNI]);
                    }
                }
            }
        }
    } else if constexpr (!(RM & 2)) {
    } else if constexpr (SPLIT) {
        if constexpr (REGS) reg_alloc<104>();
        // ------------------------------------------------------------------ epilogue warpgroups
        const int ewg = (warp - 4) / 4;        // 0..3
        const int pj = ewg / 2;                // warpgroup pair: macro tiles n = pj, pj + 2, ...
        const int h = ewg % 2;                 // column half of the macro tile
        const int q = warp % 4;                // TMEM lane quadrant
        const int r = q * 32 + lane;           // tile row == TMEM lane
        const int myhalf = r / kHalf;
        const uint32_t lane_off = (uint32_t)(q * 32) << 16;
        const float sl2 = p.scale_log2;
        int k = 0;                            // macro tiles processed by this warpgroup
        for (int n = pj;; n += 2, ++k) {
            const int buf = n % C::NACC;
            DW_WAIT(&acc_full[buf], (uint32_t)(n / C::NACC) & 1, 0);
            DW_PH0();
            tc_fence_after();
            const G1Hdr H = lds_hdr(hdr + buf);
            if (H.flags & HDR_END) break;
            // this warpgroup's 64 columns: sub-tile h (T = 64) or half h of the sub-tile (T = 128)
            const int w = (NSUB == 2 && h == 1) ? H.w1 : H.w0;
            const bool valid = w != -1 && ((tinfo_half(w) >> myhalf) & 1);
            const int c0 = tinfo_kt(w) * T + (NSUB == 1 ? 64 * h : 0);
            const int i = H.i0 + r;
            const int64_t slot = (((int64_t)H.slot_hi << 32) | (uint32_t)H.slot_lo) + (NSUB == 2 && h ? H.pad : 0);
            // one TMEM read of the row's 64 fp32 scores; the accumulator goes straight back to the MMA
            uint32_t x[64];
            if (valid) {
                tmem_ld32(tmem_base + lane_off + buf * C::MW + 64 * h, *reinterpret_cast<uint32_t(*)[32]>(&x[0]));
                tmem_ld32(tmem_base + lane_off + buf * C::MW + 64 * h + 32, *reinterpret_cast<uint32_t(*)[32]>(&x[32]));
                tmem_wait_ld();
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&acc_empty[buf]);
            DW_PH(3);
            uint8_t* stage = smem + C::OFF_X + (ewg * C::XPW + (k % C::XPW)) * C::HB;
            const uint32_t stage_s = smem_u32(stage);
            // Each warp stages and stores its own 32 rows: its slice of this staging buffer is free
            // once the warp's own store from it (XPW tiles ago) has read it.  Every warp commits one
            // bulk group per macro tile (possibly empty) so the count holds.
            if (lane == 0) {
                if (C::XPW == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
                else bulk_wait_read0();
            }
            __syncwarp();
            DW_PH(7);
            float mx = -INFINITY, dsum = 0.f;
            if (valid) {
                // mask layer: kept keys of this row form <= 2 intervals; interior
                // column ranges (every key kept) skip the bit construction entirely
                const RowMask rm = row_mask(p, i, H.kvl);
                const bool full = c0 >= rm.lo && c0 + 63 <= rm.hi &&
                                  ((c0 >= rm.blo && c0 + 63 <= rm.bhi) || c0 + 63 < rm.gc);
                if (!full) {
#pragma unroll
                    for (int c = 0; c < 2; ++c) {
                        const uint32_t bits = mask_bits32(rm, c0 + c * 32);
#pragma unroll
                        for (int u = 0; u < 32; ++u)
                            if (!((bits >> u) & 1u)) x[c * 32 + u] = 0xff800000u;  // -inf
                    }
                }
                if (LS) {
                    float m8[8];
#pragma unroll
                    for (int a = 0; a < 8; ++a) m8[a] = __uint_as_float(x[a]);
#pragma unroll
                    for (int u = 8; u < 64; ++u) m8[u & 7] = fmaxf(m8[u & 7], __uint_as_float(x[u]));
                    mx = fmaxf(fmaxf(fmaxf(m8[0], m8[1]), fmaxf(m8[2], m8[3])),
                               fmaxf(fmaxf(m8[4], m8[5]), fmaxf(m8[6], m8[7])));
                    // X' = e^{x - m'}: base 2 with log2(e) folded into the scale -- one FFMA2 per pair,
                    // then one MUFU.EX2 per element (in place)
                    const float neg = (mx == -INFINITY) ? 0.f : -mx * sl2;
#pragma unroll
                    for (int u = 0; u < 64; u += 2) {
                        float t0, t1;
                        ffma2(t0, t1, __uint_as_float(x[u]), __uint_as_float(x[u + 1]), sl2, neg);
                        float y0, y1;
#ifdef SR_DIAG_NOEXP
                        if (true) { y0 = t0; y1 = t1; } else
#endif
                        if (((u >> 1) & 7) < kPolyPairs) {
                            ex2_poly2(y0, y1, t0, t1);
                        } else {
                            y0 = ex2(t0);
                            y1 = ex2(t1);
                        }
                        x[u] = __float_as_uint(y0);
                        x[u + 1] = __float_as_uint(y1);
                    }
                    // d' = sum X' (fp32, FADD2 into 4 independent pair accumulators)
                    float sa[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll
                    for (int u = 0; u < 64; u += 2)
                        fadd2_acc(sa[(u >> 1) & 3], sa[4 + ((u >> 1) & 3)], __uint_as_float(x[u]), __uint_as_float(x[u + 1]));
                    dsum = ((sa[0] + sa[4]) + (sa[1] + sa[5])) + ((sa[2] + sa[6]) + (sa[3] + sa[7]));
                    DW_PH(4);
                } else {  // unfused baseline: the scaled, masked score
#pragma unroll
                    for (int u = 0; u < 64; u += 2) {
                        float t0, t1;
                        fmul2(t0, t1, __uint_as_float(x[u]), __uint_as_float(x[u + 1]), p.scale);
                        x[u] = __float_as_uint(t0);
                        x[u + 1] = __float_as_uint(t1);
                    }
                }
#pragma unroll
                for (int q4 = 0; q4 < 8; ++q4) {  // 8 keys -> one 16-B chunk of the fp16 tile
                    uint32_t w4[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u)
                        w4[u] = pack_f16(__uint_as_float(x[q4 * 8 + 2 * u]), __uint_as_float(x[q4 * 8 + 2 * u + 1]));
                    sts128(stage_s + tile_chunk_off(r, q4), w4[0], w4[1], w4[2], w4[3]);
                }
            }
            // the warp's 32 rows x 64 columns (4 KB, contiguous in the tile layout) go to HBM
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) {
                if (valid) {  // warp-uniform: a warp's 32 rows lie in one 64-row half
                    uint8_t* dst = (uint8_t*)p.xprime + slot * (int64_t)C::XS + (NSUB == 1 ? h * C::HB : 0) +
                                   q * 32 * 128;
                    xstore(dst, stage + q * 32 * 128, 32 * 128, (H.flags & HDR_KEEP) != 0);
                }
                bulk_commit();
            }
            DW_PH(5);
#ifdef SR_DIAG_NOSTATS
            if constexpr (false) {  // diagnostic: no statistics hand-over (timing only; results wrong)
#else
            if constexpr (IRT) {  // (m', d') of this row and sub-tile to the IR warp (-inf, 0 if invalid)
#endif
                DW_WAIT(&st_empty[buf], ((uint32_t)(n / C::NACC) & 1) ^ 1, 2);
                if (NSUB == 2 || h == 0) {
                    float* sb = stats + buf * (4 * kRowBlock) + (NSUB == 2 ? 2 * h : 0) * kRowBlock;
                    sb[r] = mx;
                    sb[kRowBlock + r] = dsum;
                }
                __syncwarp();
                if (lane == 0) mbar_arrive(&st_full[buf]);
            }
            if (LS && valid && (NSUB == 2 || h == 0)) {
                p.mprime[slot * kRowBlock + r] = mx * p.scale;  // m' in natural-log units
                if (!IRT) p.dprime[slot * kRowBlock + r] = dsum;
            }
            DW_PH(6);
        }
        if (lane == 0) bulk_wait0();
    } else {
        if constexpr (REGS) reg_alloc<224>();  // frees/takes 14336 registers, see the dealloc above
        // ------------------------------------------------------------------ epilogue warpgroups
        const int e = (warp - 4) / 4;          // warpgroup 0 / 1: even / odd macro tiles
        const int r = (warp % 4) * 32 + lane;  // tile row == TMEM lane
        const int myhalf = r / kHalf;
        const uint32_t lane_off = (uint32_t)((warp % 4) * 32) << 16;
        const float sl2 = p.scale_log2;
        const int wrow0 = (warp % 4) * 32;  // this warp's 32 rows: a contiguous 4-KB run per column half
        int k = 0;                          // macro tiles processed by this warpgroup
        // CONC: the item whose end this warp has seen but not yet announced.  It is announced one
        // header later (after that header's store group is committed, "all but the newest group
        // complete" covers every store of the item) so the X' stores overlap the next tile.
        int pend = -1;
        auto announce = [&](bool all) {
            if (lane == 0) {
                if (all) bulk_wait0();
                else asm volatile("cp.async.bulk.wait_group 1;" ::: "memory");
            }
            fence_proxy_async_global();  // this lane's m' stores before GEMM2's bulk reads of them
            __syncwarp();
            if (lane == 0) mbar_arrive(&item_done[pend % kConcNI]);
            pend = -1;
        };
        for (int n = e;; n += 2, ++k) {
            const int buf = n % C::NACC;
            DW_WAIT(&acc_full[buf], (uint32_t)(n / C::NACC) & 1, 0);
            DW_PH0();
            tc_fence_after();
            const G1Hdr H = lds_hdr(hdr + buf);
            if (H.flags & HDR_END) break;
            if constexpr (CONC) {
                if (H.flags & HDR_MARK) {  // item-end notice: release the slot, commit an empty group,
                    __syncwarp();          // pass an empty entry through the IR statistics ring
                    if (lane == 0) {
                        mbar_arrive(&acc_empty[buf]);
                        bulk_commit();
                    }
                    DW_WAIT(&st_empty[buf], ((uint32_t)(n / C::NACC) & 1) ^ 1, 2);
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&st_full[buf]);
                    if (pend >= 0) announce(false);
                    pend = H.flags >> 8;
                    if (kConcNI == 1) announce(true);  // one item in hand-over: announce at once
                    continue;
                }
            }
            const int wsub[2] = {H.w0, H.w1};
            bool vs[NSUB];  // this row's 64-row half is valid in sub-tile s
            bool any = false;
#pragma unroll
            for (int s = 0; s < NSUB; ++s) {
                vs[s] = wsub[s] != -1 && ((tinfo_half(wsub[s]) >> myhalf) & 1);
                any |= vs[s];
            }
            const int i = H.i0 + r;
            const int64_t slot = ((int64_t)H.slot_hi << 32) | (uint32_t)H.slot_lo;
            // one TMEM read of the row's MW fp32 scores; the accumulator goes straight back to the MMA
            uint32_t xr[C::MW];
            if (any) {
#pragma unroll
                for (int c = 0; c < C::MW / 32; ++c)
                    tmem_ld32(tmem_base + lane_off + buf * C::MW + c * 32, *reinterpret_cast<uint32_t(*)[32]>(&xr[c * 32]));
                tmem_wait_ld();
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&acc_empty[buf]);
            DW_PH(3);
            uint8_t* stage = smem + C::OFF_X + (e * C::XPW + (k % C::XPW)) * C::XB2;
            const uint32_t stage_s = smem_u32(stage);
            // Each warp stages and stores its own 32 rows (no warpgroup barrier): its slice of this
            // staging buffer is free once the warp's own store from it (XPW macro tiles ago) has read
            // it.  Every warp commits one bulk group per macro tile (possibly empty) so the count holds.
            if (lane == 0) {
                if (C::XPW == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
                else bulk_wait_read0();
            }
            __syncwarp();
            DW_PH(7);
            float mx[NSUB], dsum[NSUB];
            const RowMask rm = row_mask(p, i, H.kvl);
#pragma unroll
            for (int s = 0; s < NSUB; ++s) {
                mx[s] = -INFINITY;
                dsum[s] = 0.f;
                if (!vs[s]) continue;
                uint32_t* x = xr + s * T;
                const int c0 = tinfo_kt(wsub[s]) * T;
                // mask layer: kept keys of this row form <= 2 intervals; interior
                // sub-tiles (every key kept) skip the bit construction entirely
                const bool full = c0 >= rm.lo && c0 + T - 1 <= rm.hi &&
                                  ((c0 >= rm.blo && c0 + T - 1 <= rm.bhi) || c0 + T - 1 < rm.gc);
                if (!full) {
#pragma unroll
                    for (int c = 0; c < T / 32; ++c) {
                        const uint32_t bits = mask_bits32(rm, c0 + c * 32);
#pragma unroll
                        for (int u = 0; u < 32; ++u)
                            if (!((bits >> u) & 1u)) x[c * 32 + u] = 0xff800000u;  // -inf
                    }
                }
                if (LS) {
                    float m8[8];
#pragma unroll
                    for (int a = 0; a < 8; ++a) m8[a] = __uint_as_float(x[a]);
#pragma unroll
                    for (int u = 8; u < T; ++u) m8[u & 7] = fmaxf(m8[u & 7], __uint_as_float(x[u]));
                    mx[s] = fmaxf(fmaxf(fmaxf(m8[0], m8[1]), fmaxf(m8[2], m8[3])),
                                  fmaxf(fmaxf(m8[4], m8[5]), fmaxf(m8[6], m8[7])));
                    // X' = e^{x - m'}: base 2 with log2(e) folded into the scale -- one FFMA2 per pair,
                    // then one MUFU.EX2 per element (in place)
                    const float neg = (mx[s] == -INFINITY) ? 0.f : -mx[s] * sl2;
#pragma unroll
                    for (int u = 0; u < T; u += 2) {
                        float t0, t1;
                        ffma2(t0, t1, __uint_as_float(x[u]), __uint_as_float(x[u + 1]), sl2, neg);
                        float y0, y1;
#ifdef SR_DIAG_NOEXP
                        if (true) { y0 = t0; y1 = t1; } else
#endif
                        if (((u >> 1) & 7) < kPolyPairs) {
                            ex2_poly2(y0, y1, t0, t1);
                        } else {
                            y0 = ex2(t0);
                            y1 = ex2(t1);
                        }
                        x[u] = __float_as_uint(y0);
                        x[u + 1] = __float_as_uint(y1);
                    }
                    // d' = sum X' (fp32, FADD2 into 4 independent pair accumulators)
                    float sa[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll
                    for (int u = 0; u < T; u += 2)
                        fadd2_acc(sa[(u >> 1) & 3], sa[4 + ((u >> 1) & 3)], __uint_as_float(x[u]), __uint_as_float(x[u + 1]));
                    dsum[s] = ((sa[0] + sa[4]) + (sa[1] + sa[5])) + ((sa[2] + sa[6]) + (sa[3] + sa[7]));
                } else {  // unfused baseline: the scaled, masked score
#pragma unroll
                    for (int u = 0; u < T; u += 2) {
                        float t0, t1;
                        fmul2(t0, t1, __uint_as_float(x[u]), __uint_as_float(x[u + 1]), p.scale);
                        x[u] = __float_as_uint(t0);
                        x[u + 1] = __float_as_uint(t1);
                    }
                }
#pragma unroll
                for (int q4 = 0; q4 < T / 8; ++q4) {  // 8 keys -> one 16-B chunk of the fp16 tile
                    uint32_t w4[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u)
                        w4[u] = pack_f16(__uint_as_float(x[q4 * 8 + 2 * u]), __uint_as_float(x[q4 * 8 + 2 * u + 1]));
                    sts128(stage_s + tile_chunk_off(r, s * (T / 8) + q4), w4[0], w4[1], w4[2], w4[3]);
                }
            }
            DW_PH(4);
            // the warp's 32 rows of each valid sub-tile go to HBM: one 4-KB bulk copy per 64 columns
            bool wv[NSUB];
#pragma unroll
            for (int s = 0; s < NSUB; ++s) wv[s] = __shfl_sync(0xffffffffu, vs[s] ? 1 : 0, 0) != 0;
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) {
#pragma unroll
                for (int s = 0; s < NSUB; ++s) {
                    if (!wv[s]) continue;
                    uint8_t* dst = (uint8_t*)p.xprime + (slot + (s ? H.pad : 0)) * (int64_t)C::XS;
                    for (int ch = 0; ch < T / 64; ++ch)
#ifndef SR_DIAG_NOSTORE
                        xstore(dst + ch * (kRowBlock * 128) + wrow0 * 128,
                                   stage + (s * (T / 64) + ch) * (kRowBlock * 128) + wrow0 * 128, 32 * 128,
                                   (H.flags & HDR_KEEP) != 0);
#else
                        (void)dst;
#endif
                }
                bulk_commit();
            }
            DW_PH(5);
            if constexpr (IRT) {  // (m', d') of this row per sub-tile to the IR warp (-inf, 0 if invalid)
                DW_WAIT(&st_empty[buf], ((uint32_t)(n / C::NACC) & 1) ^ 1, 2);
                float* sb = stats + buf * (4 * kRowBlock);
#pragma unroll
                for (int s = 0; s < NSUB; ++s) {
                    sb[(2 * s) * kRowBlock + r] = mx[s];
                    sb[(2 * s + 1) * kRowBlock + r] = dsum[s];
                }
                __syncwarp();
                if (lane == 0) mbar_arrive(&st_full[buf]);
            }
            if (LS) {
#pragma unroll
                for (int s = 0; s < NSUB; ++s)
                    if (vs[s]) {
                        p.mprime[(slot + (s ? H.pad : 0)) * kRowBlock + r] = mx[s] * p.scale;  // natural-log units
                        if (!IRT) p.dprime[(slot + (s ? H.pad : 0)) * kRowBlock + r] = dsum[s];
                    }
            }
            DW_PH(6);
            if constexpr (CONC) {
                if (pend >= 0) announce(false);
                if (H.flags & HDR_LASTT) {
                    pend = H.flags >> 8;
                    if (kConcNI == 1) announce(true);
                }
            }
            DW_PH(1);
        }
        if (lane == 0) bulk_wait0();
        if constexpr (CONC) {
            if (pend >= 0) announce(true);
        }
    }
    DW_FLUSH(g_diag_g1);
}

}  // namespace sr
