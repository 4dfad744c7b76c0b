// tc_common.cuh -- device helpers shared by the tensor-core kernels (k_gemm1.cu, k_gemm2.cu,
// k_softmax.cu): schedule decoding, the attention-tile smem/HBM layout, interval element masks.
#pragma once
#include <climits>
#include <cstdint>

#include "ptx.cuh"
#include "sr_internal.h"

namespace sr {

constexpr int kSmemMax = 232448;  // 227 KB opt-in dynamic shared memory per CTA on sm_100
// Loads of anything a kernel of the same stream writes (the per-call schedule, kv_len, S / P / X'
// read through registers, m' / d' / r', row statistics, out / dO in the backward) are weak loads
// after griddepcontrol.wait -- __ldca (L1-cached; the GEMM kernels' schedule words) or __ldcg (L2) --
// never __ldg: every kernel is launched with programmatic dependent launch, so its CTAs may start
// before the producing kernel has written, and ld.global.nc (the read-only path, outside the memory
// model's visibility guarantees) then served stale lines even after the wait.  Found by a graph of
// eight unfused calls with different masks (tests/test_gpu_ownership.py::test_graph_capture_every_path;
// __ldca keeps the GEMMs' speed, measured: all-__ldcg cost C2 +4 %, C4 +2.5 %).  Bulk / TMA copies
// read through L2 and need no such care.
#ifndef SR_CONC_NI
#define SR_CONC_NI 2
#endif
constexpr int kConcNI = SR_CONC_NI;  // concurrent kernel (k_conc.cu): GEMM1 -> GEMM2 item hand-over ring depth

// Diagnostic build (-DSR_DIAG_WAITS, tools/diag_waits.py): every warp accumulates the clock cycles
// it spends in each class of mbarrier wait (c = 0..3) plus its lifetime (slot 4); lane 0 adds them
// to a per-kernel device array [warp][5] read back through sr_diag_read().  Off in product builds.
#ifdef SR_DIAG_WAITS
constexpr int kDW = 8;  // classes per warp (+1 lifetime slot)
#define DW_DECL long long dw_[kDW] = {}; const long long dw_start_ = clock64(); long long dw_last_ = dw_start_;
#define DW_WAIT(bar, ph, c) do { const long long t_ = clock64(); mbar_wait(bar, ph); dw_[c] += clock64() - t_; } while (0)
#define DW_TIME(stmt, c) do { const long long t_ = clock64(); stmt; dw_[c] += clock64() - t_; } while (0)
#define DW_PH0() do { dw_last_ = clock64(); } while (0)          /* start a phase sequence */
#define DW_PH(c) do { const long long t_ = clock64(); dw_[c] += t_ - dw_last_; dw_last_ = t_; } while (0)
#define DW_FLUSH(arr)                                                                                     \
    do {                                                                                                  \
        if ((threadIdx.x & 31) == 0) {                                                                    \
            const int w_ = threadIdx.x / 32;                                                              \
            for (int c_ = 0; c_ < kDW; ++c_) atomicAdd(&arr[w_ * (kDW + 1) + c_], (unsigned long long)dw_[c_]); \
            atomicAdd(&arr[w_ * (kDW + 1) + kDW], (unsigned long long)(clock64() - dw_start_));            \
        }                                                                                                 \
    } while (0)
#else
#define DW_DECL
#define DW_WAIT(bar, ph, c) mbar_wait(bar, ph)
#define DW_TIME(stmt, c) stmt
#define DW_PH0()
#define DW_PH(c)
#define DW_FLUSH(arr)
#endif

// 32-byte stage/accumulator headers are read with two ld.shared.v4 (a generic load of shared
// memory costs a long-scoreboard round trip on the consumer's critical path)
template <typename Hdr>
__device__ __forceinline__ Hdr lds_hdr(const Hdr* h)
{
    static_assert(sizeof(Hdr) == 32, "32-byte header");
    const uint32_t a = ptx::smem_u32(h);
    const uint4 x = ptx::lds128(a), y = ptx::lds128(a + 16);
    Hdr r;
    int32_t* w = reinterpret_cast<int32_t*>(&r);
    w[0] = (int32_t)x.x; w[1] = (int32_t)x.y; w[2] = (int32_t)x.z; w[3] = (int32_t)x.w;
    w[4] = (int32_t)y.x; w[5] = (int32_t)y.y; w[6] = (int32_t)y.z; w[7] = (int32_t)y.w;
    return r;
}

struct ItemInfo {
    int g, rb, t0, t1;
    int64_t slot0;  // slot id of tile t is slot0 + t
};

__device__ __forceinline__ int4 item_desc(const DevSched& sc, int it)
{
    return it < 0 ? make_int4(0, 0, 0, 0) : __ldca(sc.item_desc + it);  // precomputed on the host
}
__device__ __forceinline__ ItemInfo item_info(const DevSched& sc, int4 d)
{
    ItemInfo r;
    r.g = d.x / sc.n_rb;
    r.rb = d.x % sc.n_rb;
    r.t0 = d.y;
    r.t1 = d.z;
    r.slot0 = (int64_t)r.g * sc.slots_per_head - d.w;
    return r;
}
__device__ __forceinline__ ItemInfo decode_item(const DevSched& sc, int it) { return item_info(sc, item_desc(sc, it)); }

// Walks [it_begin, it_end) with the next item's descriptor load in flight while the current item
// runs:  for (ItemWalk w(sc, b, e); w.more(); ) { const ItemInfo I = w.next(); ... }
struct ItemWalk {
    const DevSched& sc;
    int it, begin, end;
    bool rev;  // walk [begin, end) last-first
    int4 nd;
    __device__ __forceinline__ int at(int j) const { return rev ? begin + end - 1 - j : j; }
    __device__ __forceinline__ ItemWalk(const DevSched& sc_, int b, int e, bool rev_ = false)
        : sc(sc_), it(b), begin(b), end(e), rev(rev_)
    {
        nd = item_desc(sc, it < end ? at(it) : -1);
    }
    __device__ __forceinline__ bool more() const { return it < end; }
    __device__ __forceinline__ ItemInfo next()
    {
        const ItemInfo I = item_info(sc, nd);
        ++it;
        nd = item_desc(sc, it < end ? at(it) : -1);
        return I;
    }
};

// Attention-matrix tiles (X', S, P) are 128 rows x T keys of 16-bit values in the canonical
// SWIZZLE_128B K-major layout [T/64][128 rows][64 cols]: row r of column-half h is 128 contiguous
// bytes at h*16 KB + r*128 whose 16-B chunk c sits at position c ^ (r & 7).  Byte offset of
// logical chunk c (0 .. T/8-1) of row r:
__host__ __device__ __forceinline__ uint32_t tile_chunk_off(int r, int c)
{
    return (uint32_t)((c >> 3) * (kRowBlock * 128) + r * 128 + (((c & 7) ^ (r & 7)) << 4));
}

// ---------------------------------------------------------------- element masks as intervals
// For query row i the kept keys (PAPER.md L53 mask layer) are
//     j in [lo, hi]  and  (j in [blo, bhi]  or  j < gc)
// lo/hi: key padding (kv_len) and causality; blo/bhi/gc: Longformer band and global columns
// (a global row keeps everything).  Block sparsity is handled by the tile list, not here.
struct RowMask {
    int lo, hi, blo, bhi, gc;
};

__device__ __forceinline__ RowMask row_mask(const Params& p, int i, int kvl)
{
    RowMask m;
    m.lo = 0;
    m.hi = kvl - 1;
    if (p.causal) m.hi = min(m.hi, i);
    if (p.mask_kind == MK_WINDOW && i >= p.n_global) {
        m.blo = i - p.win_half;
        m.bhi = i + p.win_half;
        m.gc = p.n_global;
    } else {
        m.blo = 0;
        m.bhi = INT_MAX / 4;
        m.gc = 0;
    }
    return m;
}

// bits u of a 32-bit word with a <= u <= b (a, b may lie outside [0, 31])
__device__ __forceinline__ uint32_t ibits32(int a, int b)
{
    a = max(a, 0);
    b = min(b, 31);
    if (b < a) return 0u;
    const uint32_t hi = (b == 31) ? 0xffffffffu : ((1u << (b + 1)) - 1u);
    const uint32_t lo = ~((1u << a) - 1u);
    return hi & lo;
}

// kept-key bits of keys c0 .. c0+31 for the row
__device__ __forceinline__ uint32_t mask_bits32(const RowMask& m, int c0)
{
    return ibits32(m.lo - c0, m.hi - c0) & (ibits32(m.blo - c0, m.bhi - c0) | ibits32(-c0, m.gc - 1 - c0));
}

}  // namespace sr
