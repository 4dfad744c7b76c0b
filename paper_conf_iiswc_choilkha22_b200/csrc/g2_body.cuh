// g2_body.cuh -- GEMM2 (device code shared by tc_gemm2 in k_gemm2.cu and the fused kernel in k_fused.cu) = Y V with the Global Scaling (GS) sub-layer fused into its prologue
// ("if element-wise scaling can be performed prior to the MatMul operation by
// providing r' corresponding to X' allocated to the TB of the MatMul kernel following the GS kernel,
// the GS kernel can easily be fused with its subsequent MatMul kernel").  GS=false builds the
// unfused baseline's GEMM2 on the softmax output P.
//
// Per item (head, 128-row block) and each of its key sub-tiles (width T):
//   Y_sub = X'_sub (fp16) * r'_row,sub (fp32), rounded once to the MMA dtype   (GS, in registers)
//   O    += Y_sub V_sub   (tcgen05.mma kind::f16, A from TMEM, B = V from smem, fp32 in TMEM)
// Macro tiles: as in GEMM1, MW = 128 keys per step -- with T = 64 two consecutive sub-tiles of the
// item (any two key blocks) are stacked along the MMA K dimension, each scaled by its own r'.
//
// Warp roles (persistent CTA per SM, 512 threads):
//   warp 0      X' producer: the macro tile's X' sub-tiles (1-D bulk copies of their valid 64-row
//               halves; the tiles are already in the UMMA SW128 K-major layout and adjacent in HBM) +
//               their r' + a stage header, into an NX-deep ring, then an END header.  The ring is only
//               read by the GS warps, so a stage is recycled once they have written it into TMEM.
//   warp 3      V producer: the macro tile's V blocks (TMA, SW128, MN-major B operand), NV-deep ring
//   warp 1      MMA issuer: per macro tile (nsub*T)/16 MMAs of 128 x D x 16 into one of two TMEM
//               O accumulators; walks the item list itself and publishes each item's output rows
//               (or EMPTY / END) to the epilogue through an O header
//   warp 2      TMEM allocator (512 columns: 2 x D for O, NA x MW/2 for the A operand ring)
//   warps 4-11  GS transform: smem X' row -> fp32 x r' -> dtype -> tcgen05.st into TMEM (A operand);
//               warp w covers TMEM lane quadrant (w-4) % 4 and key half (w-4) / 4 of each macro tile
//               (two warps per SM sub-partition: with one, GS alone bounded the kernel -- measured)
//   warps 12-15 epilogue: tcgen05.ld of O rows -> out dtype -> global
#pragma once
#include "tc_common.cuh"

namespace sr {

using namespace ptx;

#ifdef SR_DIAG_WAITS
static __device__ unsigned long long g_diag_g2[32 * (kDW + 1)];
#endif

constexpr int kMW2 = 128;  // macro tile width (keys per MMA step)
// L2 policy experiments: X' is streamed once (evict_first), V is re-read by every row-block of its
// head (evict_last); V_PREFETCH: the V producer warms the macro tile NV ahead in L2
#ifndef SR_G2_HINTS
#define SR_G2_HINTS 1
#endif
#ifndef SR_G2_VPREFETCH
#define SR_G2_VPREFETCH 0
#endif

enum : int { SH_TILE = 1, SH_END = 2, SH_EMPTY = 4, SH_FIRST = 8, SH_LAST = 16, SH_PARTIAL = 32 };
// never written: zero rows for the invalid 64-row halves of a P tile read as an smem MMA operand
static __device__ __align__(128) uint8_t g_zero_g2[kHalf * 128];
struct G2Hdr {  // X'-stage / O-buffer header
    int32_t flags, hv0, hv1, nsub, orow_lo, orow_hi, nv, pad1;  // nv: rows of the block inside the head (< 128 only
};                                                               // for the last row-block when S % 128 == 64)
// rows of row-block rb that lie inside the head (S % 128 == 64 leaves the last one half outside)
__device__ __forceinline__ int rows_in_head(const Params& p, int rb) { return min(kRowBlock, p.S - rb * kRowBlock); }

// MW_ = 64 / BUDGET / TCOLS (concurrent kernel, k_conc.cu): 64-key macro tiles in BUDGET bytes of
// shared memory and TCOLS TMEM columns (GEMM1 holds the rest of both)
template <int D, int T, int MW_ = kMW2, int BUDGET = kSmemMax, int TCOLS = 512>
struct G2 {
    static constexpr int MW = MW_;
    static constexpr int NSUB = MW / T;
    static constexpr int XS = kRowBlock * T * 2;     // X' slot (sub-tile)
    static constexpr int XB = kRowBlock * MW * 2;    // X' part of a stage (macro tile)
    static constexpr int RB = NSUB == 1 ? 1024 : 2048;  // r' (NSUB x 512 B) + header, keeps 1 KB alignment
    static constexpr int HDR_OFF = NSUB * 512;       // stage header after the r' / m' rows
    static constexpr int XSB = XB + RB;              // X' stage
    static constexpr int VB = MW * D * 2;            // V stage (macro tile)
    // split the smem budget: V stages from L2 need less depth than the HBM-bound X' stream
#ifndef SR_G2_NV64
#define SR_G2_NV64 3
#endif
#ifndef SR_G2_NV128
#define SR_G2_NV128 2
#endif
#ifndef SR_G2_NX
#define SR_G2_NX 8
#endif
    static constexpr int NV = (MW == 64 && BUDGET < kSmemMax) ? 2 : (D == 64 ? SR_G2_NV64 : SR_G2_NV128);
    static constexpr int NX_ = (BUDGET - 3072 - NV * VB) / XSB;
    static constexpr int NX = NX_ > SR_G2_NX ? SR_G2_NX : NX_;
    static_assert(NX >= 2, "smem budget");
    static constexpr int NO = 2;                             // O accumulators (D cols each)
    static constexpr int NA_ = (TCOLS - NO * D) / (MW / 2);  // A operand buffers (MW/2 cols each)
    static constexpr int NA = NA_ > 8 ? 8 : NA_;
    static_assert(NA >= 2, "tmem budget");
    static constexpr int OFF_X = 0;
    static constexpr int OFF_V = NX * XSB;
    static constexpr int OFF_BAR = OFF_V + NV * VB;
    static constexpr int NSI = 4;  // fused-IR variant: per-item (m, 1/d) row statistics in flight
    static constexpr int NBAR = 2 * NX + 2 * NV + 2 * NA + 2 * NO + 2 * NSI;
    static constexpr int OFF_STATS = OFF_BAR + NBAR * 8;                      // [NSI][2][128] fp32
    static constexpr int OFF_OHDR = OFF_STATS + NSI * 2 * kRowBlock * 4;
    static constexpr int OFF_TPTR = OFF_OHDR + NO * (int)sizeof(G2Hdr);
    static constexpr int SMEM_ = OFF_TPTR + 16 + 1024;
    static constexpr int SMEM = (BUDGET == kSmemMax && SMEM_ < 118 * 1024) ? 118 * 1024 : SMEM_;  // 1 CTA/SM
#ifndef SR_G2_NGS
#define SR_G2_NGS 8
#endif
// fp16 GS: Y = X' * r' as one mul.rn.f16x2 per pair (r' rounded to fp16 first: two roundings of
// relative 2^-11 each instead of one; r' < 2^-24 flushes to 0, a product below fp16's subnormal
// range anyway).  On by default (measured: C4 -2.2 us, C5 -1.5 us); the bf16 path goes through fp32.
#ifndef SR_G2_HMUL
#define SR_G2_HMUL 1
#endif
    static constexpr int NGS = SR_G2_NGS;       // GS warps: 8 (64 keys each) or 16 (32 keys each)
    static constexpr int KPW = MW * 4 / NGS;    // keys of a macro tile per GS warp
    static_assert(KPW % 32 == 0, "GS warp slices of whole tcgen05.st chunks");
    static constexpr int THREADS = 128 + NGS * 32 + 128;
};

// FI (fused IR): the IR sub-layer runs inside this kernel -- warp 2 reduces each
// item's m', d' into per-row (m, 1/d) ahead of the GS warps, the X' stages carry m' instead of r',
// and GS forms r' = e^{m' - m} / d on the fly.  No IR launch, no r' round trip through HBM.
// RS (default mode, IR in GEMM1): as FI, but GEMM1 already merged the rows, so warp 2 only loads each item's
// per-row (m, 1/d) -- GEMM2 applies the normalisation 1/d * e^{m' - m} in its prologue.
// Barrier initialisation of GEMM2's shared-memory layout (thread 0; fence_mbar_init included).
template <int D, int T, bool GS, bool FI, bool RS, bool AS = false, int MW = kMW2, int BUDGET = kSmemMax,
          int TCOLS = 512>
__device__ __forceinline__ void g2_init(uint8_t* smem)
{
    using C = G2<D, T, MW, BUDGET, TCOLS>;
    uint64_t* bars = (uint64_t*)(smem + C::OFF_BAR);
    uint64_t* x_full = bars;
    uint64_t* x_empty = x_full + C::NX;
    uint64_t* v_full = x_empty + C::NX;
    uint64_t* v_empty = v_full + C::NV;
    uint64_t* a_full = v_empty + C::NV;
    uint64_t* a_empty = a_full + C::NA;
    uint64_t* o_full = a_empty + C::NA;
    uint64_t* o_empty = o_full + C::NO;
    uint64_t* st_full = o_empty + C::NO;
    uint64_t* st_empty = st_full + C::NSI;
    if (threadIdx.x == 0) {
        // x_empty: the GS warps release a stage (GS), or the MMA commit (plain P . V: A read from smem)
        // (AS: the MMA commit and the NGS scaling warps, which read the stage's m')
        for (int i = 0; i < C::NX; ++i) { mbar_init(&x_full[i], 1); mbar_init(&x_empty[i], AS ? 1 + C::NGS : (GS ? C::NGS : 1)); }
        for (int i = 0; i < C::NV; ++i) { mbar_init(&v_full[i], 1); mbar_init(&v_empty[i], 1); }
        // a_full / a_empty: the TMEM A-operand ring (GS), or in AS mode the ring of per-sub-tile
        // partial products X'_k V_k (full: MMA commit; empty: the NGS scaling warps)
        for (int i = 0; i < C::NA; ++i) { mbar_init(&a_full[i], AS ? 1 : C::NGS); mbar_init(&a_empty[i], AS ? C::NGS : 1); }
        // o_full: O-header arrive + MMA commit; o_empty: one arrive per epilogue warp
        for (int i = 0; i < C::NO; ++i) { mbar_init(&o_full[i], 2); mbar_init(&o_empty[i], 4); }
        for (int i = 0; i < C::NSI; ++i) { mbar_init(&st_full[i], 1); mbar_init(&st_empty[i], C::NGS); }
        fence_mbar_init();
    }
}

// Warp roles of GEMM2 after the prologue (warps 0 .. THREADS/32 - 1; extra warps of a larger CTA idle).
// AS (accumulator-side Global Scaling, SURVEY NEXT-2's second form; fp16, requires GS, FI, RS): the
// MMA reads X' straight from its shared-memory stage (K-major SW128, invalid halves zero-filled)
// and writes each sub-tile's partial product X'_k V_k to its own TMEM buffer; the scaling warps add
// r'_k (X'_k V_k) to the rows' O in registers, r'_k = e^{m'_k - m} / d -- the same terms as
// (X'_k r'_k) V_k (Eq. 2 is linear in each sub-vector), with no per-element GS pass over X'.
// CONC (concurrent kernel, k_conc.cu): these roles run on warps WB .. WB+15 beside GEMM1's and take
// each item over from it: the X' producer and the statistics warp wait for item_done (ibar[0 ..
// kConcNI)) of every item in list order and then arrive on item_free (ibar[kConcNI ..)).
template <int D, int T, bool GS, bool FI, bool RS, bool AS = false, int MW = kMW2, int BUDGET = kSmemMax,
          int TCOLS = 512, int WB = 0, bool CONC = false, int RM = 7>
__device__ __forceinline__ void g2_roles(const CUtensorMap& tmV, const Params& p, const DevSched& sc, uint8_t* smem,
                                          uint32_t tmem_base, int it_begin, int it_end, uint64_t* ibar = nullptr)
{
    using C = G2<D, T, MW, BUDGET, TCOLS>;
    // RM: role groups compiled into this call (1: warps 0-3, 2: GS / scaling warps, 4: epilogue), so
    // a caller can run each group under its own setmaxnreg budget (k_conc.cu)
    constexpr bool R0 = RM & 1, R1 = RM & 2, R2 = RM & 4;
    static_assert(WB % 4 == 0, "TMEM lane quadrants follow warp % 4");
    static_assert(!CONC || (GS && RS && !AS), "concurrent kernel: GS prologue with GEMM1's row statistics");
    uint64_t* item_done = ibar;
    uint64_t* item_free = CONC ? ibar + kConcNI : nullptr;
    // CONC: wait until GEMM1 has completed the item at list position kord, then hand the slot back
    auto take_item = [&](int kord) {
        if constexpr (CONC) {
            mbar_wait(&item_done[kord % kConcNI], (uint32_t)(kord / kConcNI) & 1);
            __syncwarp();
            if (elect_one()) mbar_arrive(&item_free[kord % kConcNI]);
            __syncwarp();
        }
    };
    constexpr int NSUB = C::NSUB;
    uint64_t* bars = (uint64_t*)(smem + C::OFF_BAR);
    uint64_t* x_full = bars;
    uint64_t* x_empty = x_full + C::NX;
    uint64_t* v_full = x_empty + C::NX;
    uint64_t* v_empty = v_full + C::NV;
    uint64_t* a_full = v_empty + C::NV;
    uint64_t* a_empty = a_full + C::NA;
    uint64_t* o_full = a_empty + C::NA;
    uint64_t* o_empty = o_full + C::NO;
    uint64_t* st_full = o_empty + C::NO;  // fused IR: item statistics ready / consumed
    uint64_t* st_empty = st_full + C::NSI;
    float* stats = (float*)(smem + C::OFF_STATS);
    G2Hdr* ohdr = (G2Hdr*)(smem + C::OFF_OHDR);
    uint32_t* tmem_ptr = (uint32_t*)(smem + C::OFF_TPTR);
    auto xstage = [&](int s) { return smem + C::OFF_X + s * C::XSB; };
    auto xhdr = [&](int s) { return (G2Hdr*)(xstage(s) + C::XB + C::HDR_OFF); };
    auto vstage = [&](int s) { return smem + C::OFF_V + s * C::VB; };

    const int warp = warp_uniform() - WB, lane = threadIdx.x % 32;
    DW_DECL
    const uint32_t tmem_o = tmem_base;              // NO x D columns
    const uint32_t tmem_a = tmem_base + C::NO * D;  // NA x MW/2 columns
    // this CTA's items: a contiguous range of the longest-processing-time assignment (host)
    const uint8_t* src = (const uint8_t*)(GS ? p.xprime : p.pbuf);

    if (R0 && warp == 0) {
        {
            // -------------------------------------------------------------- X' producer (whole
            // warp walks the schedule; one elected lane issues)
            int s = 0;
            const uint64_t pol_x = SR_G2_HINTS ? policy_evict_first() : 0;
            uint32_t sph = 0;
            for (ItemWalk iw(sc, it_begin, it_end, p.p2_reverse); iw.more();) {
                take_item(iw.it - it_begin);  // CONC: the item's X' and m' are complete
                const ItemInfo I = iw.next();
                if (AS && I.t0 == I.t1) {  // no kept key in these rows: an EMPTY stage, written as zeros
                    DW_WAIT(&x_empty[s], sph ^ 1, 0);
                    if (elect_one()) {
                        const int64_t orow = (int64_t)I.g * p.S + I.rb * kRowBlock;
                        *xhdr(s) = G2Hdr{SH_EMPTY | SH_FIRST | SH_LAST, 0, 0, 0, (int32_t)(orow & 0xffffffff),
                                         (int32_t)(orow >> 32), rows_in_head(p, I.rb), 0};
                        mbar_arrive(&x_full[s]);
                    }
                    __syncwarp();
                    if (++s == C::NX) { s = 0; sph ^= 1; }
                    continue;
                }
                int wn[2];  // schedule words of the next macro tile, prefetched one step ahead
                for (int u = 0; u < NSUB; ++u) wn[u] = I.t0 + u < I.t1 ? __ldca(sc.tinfo + I.t0 + u) : 0;
                for (int t = I.t0; t < I.t1; t += NSUB) {
                    const int nsub = min(NSUB, I.t1 - t);
                    int hv[2] = {tinfo_half(wn[0]), NSUB > 1 ? tinfo_half(wn[1]) : 0};
                    for (int u = 0; u < NSUB; ++u) wn[u] = t + NSUB + u < I.t1 ? __ldca(sc.tinfo + t + NSUB + u) : 0;
                    uint32_t bytes = GS ? nsub * kRowBlock * 4 : 0;
#ifndef SR_DIAG2_NOX
                    for (int u = 0; u < nsub; ++u) bytes += ((GS && !AS) ? (hv[u] == 3 ? 2 : 1) : 2) * (T / 64) * (kHalf * 128);
#endif
                    DW_WAIT(&x_empty[s], sph ^ 1, 0);
                    uint8_t* st = xstage(s);
                    if (elect_one()) {
                    const int64_t orow = (int64_t)I.g * p.S + I.rb * kRowBlock;
                    *xhdr(s) = G2Hdr{SH_TILE | (t == I.t0 ? SH_FIRST : 0) | (t + NSUB >= I.t1 ? SH_LAST : 0), hv[0],
                                     hv[1], nsub, (int32_t)(orow & 0xffffffff), (int32_t)(orow >> 32),
                                     rows_in_head(p, I.rb), 0};
                    mbar_arrive_expect_tx(&x_full[s], bytes);
                    const uint8_t* xs = src + (I.slot0 + t) * (int64_t)C::XS;  // sub-tiles t, t+1 are adjacent
                    auto xload = [&](uint8_t* d, const uint8_t* g, uint32_t n) {
                        if (SR_G2_HINTS) bulk_load_hint(d, g, n, &x_full[s], pol_x);
                        else bulk_load(d, g, n, &x_full[s]);
                    };
#ifdef SR_DIAG2_NOX
                    if (false)
#endif
                    if (hv[0] == 3 && (nsub == 1 || hv[1] == 3)) {
                        xload(st, xs, nsub * C::XS);
                    } else {
                        for (int u = 0; u < nsub; ++u)
                            for (int ch = 0; ch < T / 64; ++ch) {
                                const int o = u * C::XS + ch * (kRowBlock * 128);
                                if (hv[u] == 3) xload(st + o, xs + o, kRowBlock * 128);
                                else {
                                    const int o2 = o + (hv[u] == 2 ? kHalf * 128 : 0);
                                    xload(st + o2, xs + o2, kHalf * 128);
                                    if (!GS || AS)  // the MMA reads every row of A: the invalid half is zeros
                                        bulk_load(st + (o2 ^ (kHalf * 128)), g_zero_g2, kHalf * 128, &x_full[s]);
                                }
                            }
                    }
                    if (GS)  // r' (or m' with the fused IR) of the sub-tiles' 128 rows rides along
                        bulk_load(st + C::XB, (FI ? p.mprime : p.rprime) + (I.slot0 + t) * kRowBlock,
                                  nsub * kRowBlock * 4, &x_full[s]);
                    }
                    __syncwarp();
                    if (++s == C::NX) { s = 0; sph ^= 1; }
                }
            }
            DW_WAIT(&x_empty[s], sph ^ 1, 0);
            if (elect_one()) {
                xhdr(s)->flags = SH_END;
                mbar_arrive(&x_full[s]);
            }
            __syncwarp();
        }
    } else if (R0 && warp == 2) {
        if (RS) {
            // -------------------------------------------------------------- row statistics of the
            // IR merged in GEMM1: the two partials of each of the item's 128 rows merged into (m, 1/d)
            // in the ring (lane: rows l + 32 j)
            int si = 0;
            uint32_t sph = 0;
            const int64_t nrow = (int64_t)p.B * p.H * p.Spad;  // rowstat rows: per head, whole row-blocks
            for (ItemWalk iw(sc, it_begin, it_end, p.p2_reverse); iw.more();) {
                take_item(iw.it - it_begin);  // CONC: the item's row statistics are written
                const ItemInfo I = iw.next();
                if (I.t0 == I.t1) continue;
                const int64_t row = (int64_t)I.g * p.Spad + I.rb * kRowBlock + lane;
                float mv[4], iv[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) {  // GEMM1's two IR warps' partials (m_w, d_w) of the row
                    const float ma = __ldcg(p.rowstat + row + 32 * j), da = __ldcg(p.rowstat + nrow + row + 32 * j);
                    const float mb = __ldcg(p.rowstat + 2 * nrow + row + 32 * j);
                    const float db = __ldcg(p.rowstat + 3 * nrow + row + 32 * j);
                    const float m = fmaxf(ma, mb);  // m = max_w m_w, d = sum_w e^{m_w - m} d_w
                    const float d = m == -INFINITY ? 0.f : da * __expf(ma - m) + db * __expf(mb - m);
                    mv[j] = m;
                    iv[j] = d > 0.f ? 1.f / d : 0.f;
                }
                DW_WAIT(&st_empty[si], sph ^ 1, 0);
                float* ms = stats + si * 2 * kRowBlock;
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    ms[lane + 32 * j] = mv[j];
                    ms[kRowBlock + lane + 32 * j] = iv[j];
                }
                __syncwarp();
                if (lane == 0) mbar_arrive(&st_full[si]);
                if (++si == C::NSI) { si = 0; sph ^= 1; }
            }
        } else if (FI) {
            // -------------------------------------------------------------- fused IR (NEXT-2)
            // Per non-empty item, per row: m = max_k m'_k, d = sum_k e^{m'_k - m} d'_k (PAPER.md
            // L147), published as (m, 1/d) in a ring of NSI items.  Lane l reduces rows l + 32j.
            int si = 0;
            uint32_t sph = 0;
            for (ItemWalk iw(sc, it_begin, it_end, p.p2_reverse); iw.more();) {
                const ItemInfo I = iw.next();
                if (I.t0 == I.t1) continue;
                DW_WAIT(&st_empty[si], sph ^ 1, 0);
                float* ms = stats + si * 2 * kRowBlock;
                const float* mp = p.mprime + I.slot0 * kRowBlock + lane;
                const float* dp = p.dprime + I.slot0 * kRowBlock + lane;
                float m[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY}, d[4] = {0.f, 0.f, 0.f, 0.f};
                for (int tb = I.t0; tb < I.t1; tb += 8) {
                    // one memory round trip per batch: 8 tiles x 4 rows x (m', d') + the tile words
                    float m8[4][8], d8[4][8];
                    int w8[8];
#pragma unroll
                    for (int u = 0; u < 8; ++u) w8[u] = tb + u < I.t1 ? __ldca(sc.tinfo + tb + u) : 0;
#pragma unroll
                    for (int u = 0; u < 8; ++u)
#pragma unroll
                        for (int j = 0; j < 4; ++j) {
                            const bool in = tb + u < I.t1;
                            m8[j][u] = in ? __ldca(mp + (int64_t)(tb + u) * kRowBlock + 32 * j) : -INFINITY;
                            d8[j][u] = in ? __ldca(dp + (int64_t)(tb + u) * kRowBlock + 32 * j) : 0.f;
                        }
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int half = (lane + 32 * j) / kHalf;
                        float mb = -INFINITY;
#pragma unroll
                        for (int u = 0; u < 8; ++u) {
                            if (!((tinfo_half(w8[u]) >> half) & 1) || tb + u >= I.t1) m8[j][u] = -INFINITY;
                            mb = fmaxf(mb, m8[j][u]);
                        }
                        if (mb == -INFINITY) continue;
                        const float mn = fmaxf(m[j], mb);
                        float acc = (m[j] == -INFINITY) ? 0.f : d[j] * __expf(m[j] - mn);
#pragma unroll
                        for (int u = 0; u < 8; ++u)
                            if (m8[j][u] != -INFINITY) acc += d8[j][u] * __expf(m8[j][u] - mn);
                        m[j] = mn;
                        d[j] = acc;
                    }
                }
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    ms[lane + 32 * j] = m[j];
                    ms[kRowBlock + lane + 32 * j] = d[j] > 0.f ? 1.f / d[j] : 0.f;
                }
                __syncwarp();
                if (lane == 0) mbar_arrive(&st_full[si]);
                if (++si == C::NSI) { si = 0; sph ^= 1; }
            }
        }
    } else if (R0 && warp == 3) {
        {
            // -------------------------------------------------------------- V producer (whole warp,
            // one elected lane issues)
            int s = 0;
            const uint64_t pol_v = SR_G2_HINTS ? policy_evict_last() : 0;
            uint32_t sph = 0;
            for (ItemWalk iw(sc, it_begin, it_end, p.p2_reverse); iw.more();) {
                const ItemInfo I = iw.next();
                int wn[2];  // schedule words of the next macro tile, prefetched one step ahead
                for (int u = 0; u < NSUB; ++u) wn[u] = I.t0 + u < I.t1 ? __ldca(sc.tinfo + I.t0 + u) : 0;
                for (int t = I.t0; t < I.t1; t += NSUB) {
                    const int nsub = min(NSUB, I.t1 - t);
                    int kt[2] = {tinfo_kt(wn[0]), NSUB > 1 ? tinfo_kt(wn[1]) : 0};
                    for (int u = 0; u < NSUB; ++u) wn[u] = t + NSUB + u < I.t1 ? __ldca(sc.tinfo + t + NSUB + u) : 0;
                    DW_WAIT(&v_empty[s], sph ^ 1, 0);
                    if (elect_one()) {
#ifdef SR_DIAG2_NOV
                        mbar_arrive(&v_full[s]);
                        if (false)
#else
                        mbar_arrive_expect_tx(&v_full[s], nsub * T * D * 2);
#endif
                        for (int u = 0; u < nsub; ++u)
                            for (int h = 0; h < D / 64; ++h) {
                                if (SR_G2_HINTS)
                                    tma_load_2d_hint(vstage(s) + h * (C::MW * 128) + u * (T * 128), &tmV, h * 64,
                                                     I.g * p.S + kt[u] * T, &v_full[s], pol_v);
                                else
                                    tma_load_2d(vstage(s) + h * (C::MW * 128) + u * (T * 128), &tmV, h * 64,
                                                I.g * p.S + kt[u] * T, &v_full[s]);
                            }
                        if (SR_G2_VPREFETCH) {  // the macro tile NV steps ahead in this item, into L2
                            const int tp = t + C::NV * NSUB;
                            for (int u = 0; u < NSUB; ++u)
                                if (tp + u < I.t1) {
                                    const int ktp = tinfo_kt(__ldca(sc.tinfo + tp + u));
                                    for (int h = 0; h < D / 64; ++h) tma_prefetch_2d(&tmV, h * 64, I.g * p.S + ktp * T);
                                }
                        }
                    }
                    __syncwarp();
                    if (++s == C::NV) { s = 0; sph ^= 1; }
                }
            }
        }
    } else if (AS && R0 && warp == 1) {
        // ------------------------------------------------------------------ MMA issuer (AS): per
        // macro tile and sub-tile u, X'_u V_u into the next partial-product buffer (D columns)
        const uint32_t idesc = idesc_f16(0, kRowBlock, D, 0, 1);
        int s = 0, xs = 0, j = 0;
        uint32_t sph = 0, xph = 0, jph = 0;
        for (ItemWalk iw(sc, it_begin, it_end, p.p2_reverse); iw.more();) {
            const ItemInfo I = iw.next();
            if (I.t0 == I.t1) {  // the producer posted an EMPTY stage: add our release to it
                DW_WAIT(&x_full[xs], xph, 1);
                if (elect_one()) mbar_arrive(&x_empty[xs]);
                __syncwarp();
                if (++xs == C::NX) { xs = 0; xph ^= 1; }
                continue;
            }
            for (int t = I.t0; t < I.t1; t += NSUB) {
                const int nsub = min(NSUB, I.t1 - t);
                DW_WAIT(&v_full[s], sph, 0);
                DW_WAIT(&x_full[xs], xph, 1);
                tc_fence_after();
                const uint32_t v_addr = smem_u32(vstage(s)), x_addr = smem_u32(xstage(xs));
                for (int u = 0; u < nsub; ++u) {
                    DW_WAIT(&a_empty[j], jph ^ 1, 2);
                    tc_fence_after();
                    if (elect_one()) {
#pragma unroll
                        for (int k2 = 0; k2 < T / 16; ++k2) {
                            const int kk = u * (T / 16) + k2;  // K step of 16 keys within the macro tile
                            const uint64_t bd = smem_desc_sw128(v_addr + kk * 2048, C::MW * 128, 1024);
                            const uint64_t ad = smem_desc_sw128(x_addr + (kk / 4) * (kRowBlock * 128) + (kk % 4) * 32, 16, 1024);
                            mma_ss(tmem_base + j * D, ad, bd, idesc, k2 > 0 ? 1u : 0u);
                        }
                        mma_commit(&a_full[j]);
                    }
                    __syncwarp();
                    if (++j == C::NA) { j = 0; jph ^= 1; }
                }
                if (elect_one()) {
                    mma_commit(&v_empty[s]);
                    mma_commit(&x_empty[xs]);
                }
                __syncwarp();
                if (++s == C::NV) { s = 0; sph ^= 1; }
                if (++xs == C::NX) { xs = 0; xph ^= 1; }
            }
        }
    } else if (AS && R1 && warp >= 4 && warp < 4 + C::NGS) {
        // ------------------------------------------------------------------ accumulator-side GS:
        // warp w owns TMEM lane quadrant (w-4) % 4 (32 rows) and column half (w-4) / 4 of O (D/2
        // fp32 in registers); per sub-tile u: O += r'_u * (X'_u V_u), r'_u = e^{m'_u - m} / d
        constexpr int DH = D / 2;
        const int gq = (warp - 4) % 4, hh = (warp - 4) / 4;
        const int r = gq * 32 + lane;
        const int myhalf = r / kHalf;
        const uint32_t lane_off = (uint32_t)(gq * 32) << 16;
        int s = 0, si = 0, j = 0;
        uint32_t sph = 0, siph = 0, jph = 0;
        float m_row = 0.f, invd_row = 0.f;
        float o[DH];
#pragma unroll
        for (int c = 0; c < DH; ++c) o[c] = 0.f;
        for (;;) {
            DW_WAIT(&x_full[s], sph, 0);
            const G2Hdr h = lds_hdr(xhdr(s));
            if (h.flags & SH_END) break;
            const int64_t orow = (((int64_t)h.orow_hi << 32) | (uint32_t)h.orow_lo) + r;
            if (h.flags & SH_FIRST) {
#pragma unroll
                for (int c = 0; c < DH; ++c) o[c] = 0.f;
                if (!(h.flags & SH_EMPTY)) {  // the statistics warp skips empty items
                    DW_WAIT(&st_full[si], siph, 2);
                    m_row = stats[si * 2 * kRowBlock + r];
                    invd_row = stats[si * 2 * kRowBlock + kRowBlock + r];
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&st_empty[si]);
                    if (++si == C::NSI) { si = 0; siph ^= 1; }
                }
            }
            if (!(h.flags & SH_EMPTY)) {
                const uint32_t xs_s = smem_u32(xstage(s));
                const int hvs[2] = {h.hv0, h.hv1};
                float rr[NSUB];
#pragma unroll
                for (int u = 0; u < NSUB; ++u) {
                    const bool valid = u < h.nsub && ((hvs[u] >> myhalf) & 1);
                    const float mp = valid ? lds_f32(xs_s + C::XB + u * 512 + 4 * r) : -INFINITY;
                    rr[u] = (mp == -INFINITY) ? 0.f : __expf(mp - m_row) * invd_row;  // 0 for a masked sub-vector
                }
                __syncwarp();
                if (lane == 0) mbar_arrive(&x_empty[s]);  // m' read; the MMA commit releases the X' data
#pragma unroll
                for (int u = 0; u < NSUB; ++u) {
                    if (u >= h.nsub) break;
                    DW_WAIT(&a_full[j], jph, 1);
                    tc_fence_after();
#pragma unroll
                    for (int c = 0; c < DH / 32; ++c) {
                        uint32_t v[32];
                        tmem_ld32(tmem_base + lane_off + j * D + hh * DH + c * 32, v);
                        tmem_wait_ld();
#pragma unroll
                        for (int i = 0; i < 32; ++i) o[c * 32 + i] = fmaf(rr[u], __uint_as_float(v[i]), o[c * 32 + i]);
                    }
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&a_empty[j]);
                    if (++j == C::NA) { j = 0; jph ^= 1; }
                }
            } else {
                __syncwarp();
                if (lane == 0) mbar_arrive(&x_empty[s]);
            }
            if ((h.flags & SH_LAST) && r < h.nv) {  // this warp's D/2 columns of its 32 output rows
                if (p.out_dtype == DT_F32) {
                    float4* O = reinterpret_cast<float4*>((float*)p.out + orow * D + hh * DH);
#pragma unroll
                    for (int c = 0; c < DH / 4; ++c) O[c] = make_float4(o[4 * c], o[4 * c + 1], o[4 * c + 2], o[4 * c + 3]);
                } else {
                    uint4* O = reinterpret_cast<uint4*>((uint16_t*)p.out + orow * D + hh * DH);
#pragma unroll
                    for (int c = 0; c < DH / 8; ++c)
                        O[c] = make_uint4(pack_f16(o[8 * c], o[8 * c + 1]), pack_f16(o[8 * c + 2], o[8 * c + 3]),
                                          pack_f16(o[8 * c + 4], o[8 * c + 5]), pack_f16(o[8 * c + 6], o[8 * c + 7]));
                }
            }
            if (++s == C::NX) { s = 0; sph ^= 1; }
        }
    } else if (R0 && warp == 1) {
        {
            // -------------------------------------------------------------- MMA issuer (whole warp,
            // one elected lane issues)
            const uint32_t idesc = idesc_f16(p.in_dtype == DT_BF16 ? 1 : 0, kRowBlock, D, 0, 1);
            int s = 0, a = 0, o = 0, xs = 0;
            uint32_t sph = 0, aph = 0, oph = 0, xph = 0;
            auto post = [&](int flags, int64_t orow, int nv, bool second) {  // O header, arrival 1 of 2
                DW_WAIT(&o_empty[o], oph ^ 1, 2);
                if (elect_one()) {
                    ohdr[o] = G2Hdr{flags, 0, 0, 0, (int32_t)(orow & 0xffffffff), (int32_t)(orow >> 32), nv, 0};
                    mbar_arrive(&o_full[o]);
                    if (second) mbar_arrive(&o_full[o]);  // no MMA commit will follow
                }
                __syncwarp();
            };
            auto next_o = [&]() {
                if (++o == C::NO) { o = 0; oph ^= 1; }
            };
            ItemInfo nxt;
            auto at = [&](int j) { return p.p2_reverse ? it_begin + it_end - 1 - j : j; };
            if (it_begin < it_end) nxt = decode_item(sc, at(it_begin));
            for (int it = it_begin; it < it_end; ++it) {
                const ItemInfo I = nxt;
                if (it + 1 < it_end) nxt = decode_item(sc, at(it + 1));  // prefetch
                // a chunk of a split row-block (SR_SPLIT_KV) writes fp32 partial rows to its slot
                const int ps = (!AS && p.partial) ? __ldca(sc.psl + at(it)) : -1;
                const int64_t orow = ps >= 0 ? (int64_t)ps * kRowBlock : (int64_t)I.g * p.S + I.rb * kRowBlock;
                const int nv = ps >= 0 ? kRowBlock : rows_in_head(p, I.rb);  // a partial slot holds all 128
                if (I.t0 == I.t1) {  // no kept key in these rows: the epilogue writes zeros
                    post(SH_EMPTY, orow, nv, true);
                    next_o();
                    continue;
                }
                post(SH_TILE | (ps >= 0 ? SH_PARTIAL : 0), orow, nv, false);
                const uint32_t d_tmem = tmem_o + o * D;
                for (int t = I.t0; t < I.t1; t += NSUB) {
                    const int nk = min(NSUB, I.t1 - t) * (T / 16);  // K steps of 16 keys
                    DW_WAIT(&v_full[s], sph, 0);
                    if (GS) DW_WAIT(&a_full[a], aph, 1);
                    else DW_WAIT(&x_full[xs], xph, 1);
                    tc_fence_after();
                    const uint32_t v_addr = smem_u32(vstage(s));
                    const uint32_t a_tm = tmem_a + a * (C::MW / 2);
                    const uint32_t x_addr = smem_u32(xstage(xs));
                    if (elect_one()) {
#pragma unroll 8
                        for (int kk = 0; kk < nk; ++kk) {
                            // B = V, MN-major SW128: 16 keys per MMA = 2 KB; 64-wide d blocks at LBO = MW*128 B
                            const uint64_t bd = smem_desc_sw128(v_addr + kk * 2048, C::MW * 128, 1024);
                            if (GS) {
                                mma_ts(d_tmem, a_tm + kk * 8, bd, idesc, (t == I.t0 && kk == 0) ? 0u : 1u);
                            } else {  // A = the P tile in the stage: K-major SW128, 64-key blocks 16 KB apart
                                const uint64_t ad = smem_desc_sw128(x_addr + (kk / 4) * (kRowBlock * 128) + (kk % 4) * 32, 16, 1024);
                                mma_ss(d_tmem, ad, bd, idesc, (t == I.t0 && kk == 0) ? 0u : 1u);
                            }
                        }
                        mma_commit(&v_empty[s]);
                        if (GS) mma_commit(&a_empty[a]);
                        else mma_commit(&x_empty[xs]);
                    }
                    __syncwarp();
                    if (++s == C::NV) { s = 0; sph ^= 1; }
                    if (GS) { if (++a == C::NA) { a = 0; aph ^= 1; } }
                    else if (++xs == C::NX) { xs = 0; xph ^= 1; }
                }
                if (elect_one()) mma_commit(&o_full[o]);  // arrival 2 of 2 when the item's MMAs complete
                __syncwarp();
                next_o();
            }
            post(SH_END, 0, 0, true);
        }
    } else if (GS && !AS && R1 && warp >= 4 && warp < 4 + C::NGS) {
        // ------------------------------------------------------------------ GS transform
        const int gq = (warp - 4) % 4, ch = (warp - 4) / 4;  // lane quadrant, key slice (KPW keys)
        constexpr int KPW = C::KPW;
        const int r = gq * 32 + lane;
        const int myhalf = r / kHalf;
        const uint32_t lane_off = (uint32_t)(gq * 32) << 16;
        const bool bf = p.in_dtype == DT_BF16;
        int s = 0, a = 0, si = 0;
        uint32_t sph = 0, aph = 0, siph = 0;
        float m_row = 0.f, invd_row = 0.f;  // fused IR: this row's (m, 1/d) for the current item
        for (;;) {
            DW_WAIT(&x_full[s], sph, 0);
            const G2Hdr h = lds_hdr(xhdr(s));
            if (h.flags & SH_END) break;
            if (FI && (h.flags & SH_FIRST)) {  // a new item: its row statistics from the IR warp
                DW_WAIT(&st_full[si], siph, 2);
                m_row = stats[si * 2 * kRowBlock + r];
                invd_row = stats[si * 2 * kRowBlock + kRowBlock + r];
                __syncwarp();
                if (lane == 0) mbar_arrive(&st_empty[si]);
                if (++si == C::NSI) { si = 0; siph ^= 1; }
            }
            const uint32_t xs_s = smem_u32(xstage(s));
            const int hvs[2] = {h.hv0, h.hv1};
            float rr[NSUB];
#pragma unroll
            for (int u = 0; u < NSUB; ++u) {
                const bool valid = u < h.nsub && ((hvs[u] >> myhalf) & 1);
                rr[u] = valid ? 1.f : 0.f;
                if (GS && valid) {
                    const float v = lds_f32(xs_s + C::XB + u * 512 + 4 * r);
                    if (FI)  // r'_k = e^{m'_k - m} / d  (0 for a fully masked sub-vector)
                        rr[u] = (v == -INFINITY) ? 0.f : __expf(v - m_row) * invd_row;
                    else
                        rr[u] = v;
                }
            }
            uint32_t rh[NSUB];  // r' as f16x2 (fp16 fast path)
#pragma unroll
            for (int u = 0; u < NSUB; ++u) rh[u] = pack_f16(rr[u], rr[u]);
            // this warp's slice of the X' row (KPW fp16 = KPW/8 chunks of 16 B) into registers first:
            // the loads overlap the wait for a free A buffer
            uint4 xv[KPW / 8];
#ifdef SR_DIAG2_NOGS
            if (false)
#endif
#pragma unroll
            for (int q = 0; q < KPW / 8; ++q)  // unconditional: issued beside the r' chain (unused if r' = 0)
                xv[q] = lds128(xs_s + tile_chunk_off(r, ch * (KPW / 8) + q));
            DW_WAIT(&a_empty[a], aph ^ 1, 1);
            tc_fence_after();
            const uint32_t a_tm = tmem_a + lane_off + a * (C::MW / 2);
#pragma unroll
            for (int c2 = 0; c2 < KPW / 32; ++c2) {  // 32 keys -> 16 packed words per tcgen05.st
                const int c = ch * (KPW / 32) + c2;
                const int u = (c * 32) / T;   // sub-tile of these keys
                uint32_t pk[16];
                if (rr[u] != 0.f) {
#pragma unroll
                    for (int q4 = 0; q4 < 4; ++q4) {
                        const uint4 x = xv[c2 * 4 + q4];
                        const uint32_t xw[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
                        for (int w = 0; w < 4; ++w) {
                            if (GS && SR_G2_HMUL && !bf) {  // fp16: one packed f16x2 multiply per pair
                                uint32_t y;
                                asm("mul.rn.f16x2 %0, %1, %2;" : "=r"(y) : "r"(xw[w]), "r"(rh[u]));
                                pk[q4 * 4 + w] = y;
                            } else if (GS) {  // Y = X' * r'  (fp16 X' -> fp32 -> x r' -> dtype, one rounding)
                                const float2 f = unpack_f16(xw[w]);
                                float y0, y1;
                                fmul2(y0, y1, f.x, f.y, rr[u]);
                                pk[q4 * 4 + w] = bf ? pack_bf16(y0, y1) : pack_f16(y0, y1);
                            } else {  // P already holds dtype values
                                pk[q4 * 4 + w] = xw[w];
                            }
                        }
                    }
                } else {  // absent sub-tile, invalid half (not loaded) or r' = 0: zero rows of A
#pragma unroll
                    for (int w = 0; w < 16; ++w) pk[w] = 0u;
                }
#ifndef SR_DIAG2_NOGS
                tmem_st16(a_tm + c * 16, pk);
#else
                (void)pk;
#endif
            }
            tmem_wait_st();
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&a_full[a]);
            if (++a == C::NA) { a = 0; aph ^= 1; }
            // release the X' stage only now: its ld.shared results have been consumed by the tcgen05.st
            // above.  Arriving right after issuing the loads let the next bulk copy overwrite the stage
            // while other lanes' loads were still in flight (a real race, seen as 16-lane corruption).
            if (lane == 0) mbar_arrive(&x_empty[s]);
            if (++s == C::NX) { s = 0; sph ^= 1; }
        }
    } else if (!AS && R2 && warp >= 4 + C::NGS && warp < 8 + C::NGS) {
        // ------------------------------------------------------------------ output epilogue
        const int r = (warp % 4) * 32 + lane;
        const uint32_t lane_off = (uint32_t)((warp % 4) * 32) << 16;
        int o = 0;
        uint32_t oph = 0;
        for (;;) {
            DW_WAIT(&o_full[o], oph, 0);
            tc_fence_after();
            const G2Hdr h = lds_hdr(ohdr + o);
            if (h.flags & SH_END) break;
            const int64_t orow = (((int64_t)h.orow_hi << 32) | (uint32_t)h.orow_lo) + r;
            if (h.flags & SH_EMPTY) {  // no kept key anywhere in these rows: output 0 (reading R9)
                if (r >= h.nv) {       // (a row beyond the head: not ours to write)
                } else if (p.out_dtype == DT_F32) {
                    float4* O = reinterpret_cast<float4*>((float*)p.out + orow * D);
                    for (int c = 0; c < D / 4; ++c) O[c] = make_float4(0.f, 0.f, 0.f, 0.f);
                } else {
                    uint4* O = reinterpret_cast<uint4*>((uint16_t*)p.out + orow * D);
                    for (int c = 0; c < D / 8; ++c) O[c] = make_uint4(0, 0, 0, 0);
                }
            } else {
                const uint32_t taddr = tmem_o + lane_off + o * D;
                const bool part = (h.flags & SH_PARTIAL) != 0;  // fp32 partial rows of a split row-block
#pragma unroll
                for (int c = 0; c < D / 32; ++c) {
                    uint32_t v[32];
                    tmem_ld32(taddr + c * 32, v);
                    tmem_wait_ld();
                    if (r >= h.nv) {  // a row beyond the head (S % 128 == 64): loaded with the warp, not stored
                    } else if (part || p.out_dtype == DT_F32) {
                        float4* O = reinterpret_cast<float4*>((part ? p.partial : (float*)p.out) + orow * D + c * 32);
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
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&o_empty[o]);
            if (++o == C::NO) { o = 0; oph ^= 1; }
        }
    }
    DW_FLUSH(g_diag_g2);
}

}  // namespace sr
