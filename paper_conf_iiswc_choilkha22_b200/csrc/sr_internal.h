// sr_internal.h -- shared declarations of the sr_mha library (host + device).  Not installed.
//
// Terminology:
//   row-block  128 consecutive query rows of one head (the M = 128 tcgen05 tile)
//   key tile   T consecutive keys (T = LS sub-vector width = GEMM1 output-tile width)
//   tile       (head, row-block, key tile); its two 64-row halves can be valid independently
//              (block-sparse pairs of 64-row block-rows, causal diagonals with T = 64, band edges)
//   slot       storage index of a tile inside the workspace: X' tile, and 128 m'/d'/r' floats
//   item       (head, row-block): the unit of work of the GEMM kernels, scheduled longest-first
#pragma once
#include <cstddef>
#include <cstdint>
#include <cstdlib>

#include <cuda_runtime.h>

#include <utility>

namespace sr {

constexpr int kRowBlock = 128;  // M of every tcgen05 tile
constexpr int kHalf = 64;       // validity granularity of tile rows
#ifndef SR_IR_WARP_TILES
#define SR_IR_WARP_TILES 4
#endif
// IR kernel: tiles one warp merges in registers (4: 80 registers, three 8-warp CTAs per SM; 8 held
// 122 registers and ran C4's row-blocks in two waves; a form staging the statistics in shared memory
// by bulk copies was slower back to back -- measured, profiles/r2_experiments.txt).  kIrWarpTilesWide
// (6, still three CTAs per SM) is taken when the 4-tile classes would need more than one wave of
// CTAs: fewer, wider teams then run in one wave (C4 6.76 -> 6.14 us back to back).
constexpr int kIrWarpTilesWide = 6;
constexpr int kIrCtasPerSm = 3;
constexpr int kIrWarpTiles = SR_IR_WARP_TILES;
constexpr int kSplitRefSms = 148; // SR_SPLIT_KV chunk size reference: about two chunks per SM of a B200
constexpr int kSmShortChunks = 16; // unfused softmax: rows of up to this many 64-key chunks form the short class

// Where the IR sub-layer runs: its own kernel (SR_IR_KERNEL, the paper's layout), folded into
// GEMM2 (SR_FUSE_IR), or merged by warps of GEMM1 as the row's tiles are produced (default).
enum IrMode : int { IR_KERNEL = 0, IR_IN_GEMM2 = 1, IR_IN_GEMM1 = 2 };
enum MaskKind : int { MK_DENSE = 0, MK_BLOCK = 1, MK_WINDOW = 2 };
enum DType : int { DT_F32 = 0, DT_F16 = 1, DT_BF16 = 2 };
// lh_mode: which layout list a head g = b*H + h uses
enum LhMode : int { LH_ONE = 0, LH_BATCH = 1, LH_HEAD = 2 };

// tile info word: key-tile index in units of T (bits 0-15) | half-valid bits (16: rows 0-63,
// 17: rows 64-127)
__host__ __device__ inline int tinfo_kt(int32_t w) { return w & 0xFFFF; }
__host__ __device__ inline int tinfo_half(int32_t w) { return (w >> 16) & 3; }

// Device-side view of a cached schedule.
struct DevSched {
    const int32_t* tp;      // [n_lh][n_rb+1] absolute offsets into tinfo
    const int32_t* tinfo;   // [n_tiles_list]
    const int32_t* items;   // [n_items] g * n_rb + rb; grouped by persistent CTA, longest first
    const int32_t* cta_ptr; // [n_cta + 1]: CTA c runs items[cta_ptr[c] .. cta_ptr[c+1])
    const int4* item_desc;  // [n_items] {item, t0, t1, tp[lh][0]}: one 16-B load per item decode
    // GEMM1 pair schedule (row-blocks 2j, 2j+1 share K tiles): pair items {g * n_pair + j, e0, e1,
    // tp[lh][0]} grouped per CTA by pcta_ptr; pent[e] = {kt | ha << 16 | hb << 18, ta, tb, 0}
    const int4* pair_desc;
    const int4* pent;
    const int32_t* pcta_ptr;
    int n_pair, n_pcta;
    // the same pair assignment as row-block items (one-launch kernel with pairs: phase 2 walks the
    // row-blocks its phase 1 produced): fp_desc in item_desc format, grouped per CTA by fpcta_ptr
    const int4* fp_desc;
    const int32_t* fpcta_ptr;
    const int32_t* kv_len;  // [B] or nullptr
    int n_rb, n_lh, lh_mode, slots_per_head, n_items, n_cta;
    int max_rb_tiles;       // longest tile list of one (layout head, row-block)
    int mean_rb_tiles;      // mean tile-list length, rounded up
    // column schedule (training backward, dK / dV): column items = (head, 128-key column block c),
    // col_desc[i] = {g * n_cb + c, e0, e1, tp[lh][0]} grouped per CTA by ccta_ptr; cent[e] =
    // {rb | half bits of key tile a << 16 | of key tile b << 18, tinfo index of a or -1, of b or -1, 0}
    // with a, b the key tiles 2c, 2c+1 (T = 64) or a = c alone (T = 128), row-blocks ascending
    const int4* col_desc;
    const int4* cent;
    const int32_t* ccta_ptr;
    int n_cb, n_ccta;
    // standalone IR kernel (SR_IR_KERNEL): row-blocks longest first, in classes of team size 8, 4, 2, 1
    // warps (> 4, 2, 1 x ir_warp_tiles tiles, the rest); n_ir_class[c] row-blocks in class c
    const int4* ir_desc;  // {g * slots_per_head + t0 - tp[lh][0], t1 - t0, t0, item} per row-block, class order
    int n_ir_class[4];
    int ir_warp_tiles;  // kIrWarpTiles or kIrWarpTilesWide: the tiles per warp the classes were cut for
    int simt_tpr;       // fp32 SIMT kernels: threads per query row (4, 8, 16, 32; k_simt_f32.cu)
    // key-range split (SR_SPLIT_KV): psl[i] = partial-output slot of item descriptor i (a chunk of a
    // split row-block) or -1; comb[j] = {row-block item, first slot, chunks, 0} of split row-block j
    const int32_t* psl;
    const int4* comb;
    int n_comb;
    // unfused softmax: 64-row halves whose rows exceed kSmShortChunks chunks, (item * 2 + half)
    const int32_t* sm_long;
    int n_sm_long;
};

// Everything a kernel needs to know about one call.
struct Params {
    const void* q;
    const void* k;
    const void* v;
    void* out;
    int B, H, S, D, T;
    int Spad;          // S rounded up to whole 128-row blocks: the per-head stride of rowstat / bstat
    float scale;       // multiplies Q K^T
    float scale_log2;  // scale * log2(e): the GEMM1 epilogue works in base 2
    int causal;
    int mask_kind;     // MaskKind (element masks: kv_len, causal, window; blocks come from tinfo)
    int win_half;      // window / 2
    int n_global;
    int in_dtype, out_dtype;
    int stages;        // SR_RUN_* bits to launch
    int ir_mode;       // IrMode: where the IR sub-layer runs
    int g1_pair;       // GEMM1 walks pairs of row-blocks sharing each K tile (pair schedule)
    int gs_prologue;   // one-launch kernel: Global Scaling in GEMM2's prologue even for fp16 (SR_GS_PROLOGUE)
    int x_evict_first; // GEMM1's X' / S tile stores carry an L2 evict_first policy (large layers only)
    int x_keep;        // one-launch kernel: the last x_keep items of each CTA store X' at normal L2 priority ...
    int p2_reverse;    // ... and phase 2 walks the CTA's items last-first, reading that X' back from L2
    int p1_reverse;    // one-launch kernel: phase 1 walks the CTA's items last-first (phase 2 then forward)
    DevSched sc;
    void* xprime;      // X' tiles (recomposed) or score tiles S (unfused)
    void* pbuf;        // unfused: P tiles
    float* mprime;
    float* dprime;
    float* rprime;
    float* rowstat;    // IR_IN_GEMM1: [2 partials][m (natural log) | d][B*H*S] per query row
    // training backward (NEXT-4)
    const void* dout;  // dE/dO [B,H,S,D], in_dtype
    void* dq;          // gradients [B,H,S,D], out_dtype
    void* dk;
    void* dv;
    void* dsbuf;       // dS' = scale * dE/dx tiles (in_dtype), same slots and layout as X'
    float* bstat;      // [3][B*H*S]: per query row m (natural log), 1/d, delta = sum_d dO * O
    float* partial;    // SR_SPLIT_KV: fp32 [slot][128][D] partial outputs of split row-blocks' chunks
    int bwd_dq_fused;  // dQ accumulated inside the dS' kernel (default; SR_BWD_DQ_SEPARATE=1: own kernel)
};

__host__ __device__ inline int lh_of(const DevSched& s, int g, int H)
{
    return s.lh_mode == LH_ONE ? 0 : (s.lh_mode == LH_BATCH ? g / H : g % H);
}

// Element mask: kept iff every active criterion keeps (i, j).  Block-level
// sparsity is not evaluated here: it is encoded in the tile list / half bits.
__host__ __device__ inline bool elem_kept(const Params& p, int kvl, int i, int j)
{
    if (j >= kvl) return false;
    if (p.causal && j > i) return false;
    if (p.mask_kind == MK_WINDOW) {
        int dd = i - j;
        dd = dd < 0 ? -dd : dd;
        if (!(dd <= p.win_half || i < p.n_global || j < p.n_global)) return false;
    }
    return true;
}

// Launch with Programmatic Dependent Launch enabled: the kernel may begin (prologue) while the
// previous kernel in the stream drains; it must call griddepcontrol.wait before reading results of
// that kernel (all sr kernels do).
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                              int64_t* nlaunch, Args&&... args)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    static const bool no_pdl = getenv("SR_NO_PDL") != nullptr;  // experiments: plain stream order
    cfg.numAttrs = no_pdl ? 0 : 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
    ++*nlaunch;
    return e != cudaSuccess ? e : cudaGetLastError();
}

// ---- launchers (return cudaError_t of the launch)
cudaError_t launch_simt_f32(const Params& p, cudaStream_t st, int64_t* nlaunch);
cudaError_t launch_ir(const Params& p, cudaStream_t st, int64_t* nlaunch);
cudaError_t launch_combine(const Params& p, cudaStream_t st, int64_t* nlaunch);
cudaError_t launch_tc_fused(const Params& p, cudaStream_t st, int64_t* nlaunch);
cudaError_t launch_tc_unfused(const Params& p, cudaStream_t st, int64_t* nlaunch);
cudaError_t launch_tc_sd(const Params& p, cudaStream_t st, int64_t* nlaunch);
cudaError_t launch_tc_bwd(const Params& p, cudaStream_t st, int64_t* nlaunch);
cudaError_t launch_tc_one(const Params& p, cudaStream_t st, int64_t* nlaunch);
cudaError_t launch_tc_conc(const Params& p, cudaStream_t st, int64_t* nlaunch);
// k_sched.cu: enqueue copies of n_seg word ranges [seg_off, seg_off + seg_len) of `words` (int32
// offsets / lengths, multiples of 4) into the same offsets of `region` (device, 16-B aligned),
// carried in kernel parameters
cudaError_t launch_sched_upload(void* region, const int32_t* words, const size_t* seg_off, const size_t* seg_len,
                                int n_seg, cudaStream_t st, int64_t* nlaunch);

}  // namespace sr
