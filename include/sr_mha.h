/*
 * sr_mha.h -- C ABI of the B200-native softmax-recomposed multi-head attention hot path.
 *
 * Method: Choi, Li, Kim, Hwang, Ahn, "Accelerating Transformer Networks through Recomposing
 * Softmax Layers", IISWC 2022.  The attention layer computes, per
 * head, O = softmax(mask(Q K^T * scale)) V with the safe softmax of Eq. (1) (L55-L58).  This
 * library computes it through the paper's softmax recomposition (Sec. 3.2-3.4):
 *
 *   kernel 1  GEMM1 + LS   x = Q K^T * scale, mask; per 128-row x T-column output tile the
 *             (+ IR)       epilogue computes the Local Softmax (Eq. 2): m' = row max of the tile,
 *                          X' = e^{x - m'} (written once), d' = row sum of X'     (L131-L145, L165).
 *                          The Inter-sub-vector Reduction runs in the same kernel: a GEMM1 CTA owns
 *                          whole rows, so two of its warps merge each row's (m'_k, d'_k) as they are
 *                          produced: m = max_k m'_k, d = sum_k e^{m'_k - m} d'_k  (L147-L149)
 *   kernel 2  GS + GEMM2   the prologue scales each X' tile row by r'_k = e^{m'_k - m} / d (Global
 *                          Scaling, L151) as the tile is loaded, then O += Y V on the tensor cores
 *
 * By default (16-bit) both kernels' work runs in ONE launch: each CTA does kernel 1 for its rows,
 * then kernel 2 for the same rows (SR_ONE_KERNEL below); SR_TWO_KERNELS launches them separately.
 * The paper's own layout -- IR as a third, standalone kernel writing r' (L173) -- is the
 * SR_IR_KERNEL variant; SR_FUSE_IR and SR_DECOMPOSE are the other variants (see below).
 *
 * The attention matrix therefore crosses HBM twice instead of four times (L171-L173).  The
 * *_unfused entry points run the deliberately unfused baseline GEMM1 -> row softmax -> GEMM2
 * (L102, L171) with the same tiles, skipping and layouts, as the in-repo traffic baseline.
 *
 * Conventions common to every entry point
 * ---------------------------------------
 *  - q, k, v, out: DEVICE pointers, [B][H][S][D] contiguous (the caller does the Split/Concat of
 *    PAPER.md L49-L51), 16-byte aligned.  in_dtype for q/k/v; out_dtype for out.  out is fully
 *    overwritten and must not overlap q, k or v.
 *  - scale: multiplies Q K^T (PAPER.md L53 uses 1/sqrt(D_head)); finite and > 0.
 *  - causal: key j is masked for query i when j > i (combines with every mask kind).
 *  - Mask / layout descriptors and the arrays they point to are HOST memory, read during the
 *    call (they may be freed or changed once the call returns).  The library derives a tile
 *    schedule from them on the host, keeps it in a bounded host-side cache keyed by the mask
 *    content, and every call writes it into the caller's workspace (region off_sched) with a
 *    stream-ordered copy kernel whose words travel in its launch parameters.
 *  - Ownership: the caller owns q, k, v, out, the workspace, the mask arrays and the stream.  The
 *    library never allocates device memory and never synchronises: every call -- including the
 *    first call with a new mask -- only enqueues kernels on ex->stream, so any call can be captured
 *    in a CUDA graph, and a replay is self-contained (it re-writes the schedule it captured).
 *    Calls are asynchronous: device-side faults surface at the caller's next synchronisation (as
 *    with cuBLAS).  Two calls in flight at once (other streams, other threads) need two workspaces.
 *  - A row whose every key is masked outputs 0 (reading R9).
 *  - Supported: S % 64 == 0, S >= 64 (tile_n = 128 needs S % 128 == 0; with S % 128 == 64 the default
 *    sub-vector is 64 and the last 128-row tile is half inside the head -- its other half is never
 *    computed into the workspace and no row beyond S of out / dq / dk / dv is written);
 *    D in {64, 128}; in_dtype F16 or BF16 (tensor-core path) or
 *    F32 (SIMT fp32 path, every mask kind); out_dtype == in_dtype or F32; block == 64.
 *    Anything else returns SR_ERR_UNSUPPORTED before touching the device.
 *
 * Errors: argument checks run before any CUDA call and return SR_ERR_INVALID /
 * SR_ERR_UNSUPPORTED / SR_ERR_WORKSPACE; a failed CUDA call returns SR_ERR_CUDA.  Details of the
 * last non-OK return on the calling thread: sr_last_error().
 */
#ifndef SR_MHA_H
#define SR_MHA_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    SR_OK = 0,
    SR_ERR_INVALID = 1,     /* bad pointer, shape, scale, overlapping out, malformed layout */
    SR_ERR_UNSUPPORTED = 2, /* valid request outside the supported envelope (see above) */
    SR_ERR_WORKSPACE = 3,   /* workspace NULL or smaller than sr_workspace_bytes() */
    SR_ERR_CUDA = 4         /* a CUDA runtime/driver call failed; see sr_last_error() */
} sr_status;

typedef enum { SR_F32 = 0, SR_F16 = 1, SR_BF16 = 2 } sr_dtype;

/* Dense mask: optional key-side padding.  kv_len: HOST array [B] or NULL;
 * key j of batch b is masked iff j >= kv_len[b]  (0 <= kv_len[b] <= S). */
typedef struct {
    const int32_t* kv_len;
} sr_dense_mask;

/* Block-sparse layout (square blocks).  HOST arrays.
 *   block         block edge, must be 64
 *   layout_heads  1 (shared by all heads) or H (head h uses layout h, for every batch b)
 *   row_ptr       [layout_heads][S/block + 1]: ABSOLUTE offsets into col_idx; row_ptr[h][0] is the
 *                 start of head h, non-decreasing
 *   col_idx       column-block ids, strictly ascending within a block-row, in [0, S/block)
 * Element (i, j) is kept iff block (i/64, j/64) is listed (and causal allows it). */
typedef struct {
    int32_t block;
    int32_t layout_heads;
    const int32_t* row_ptr;
    const int32_t* col_idx;
} sr_block_layout;

/* Longformer sliding window + symmetric global tokens:
 * (i, j) kept iff |i - j| <= window/2  or  i < n_global  or  j < n_global. */
typedef struct {
    int32_t window;
    int32_t n_global;
} sr_window;

/* Execution parameters. */
typedef struct {
    sr_dtype in_dtype;       /* dtype of q, k, v */
    sr_dtype out_dtype;      /* in_dtype, or SR_F32 (fp32-accumulated context, validation mode) */
    void* workspace;         /* DEVICE, caller-owned, >= sr_workspace_bytes(), 256-byte aligned */
    size_t workspace_bytes;
    void* stream;            /* cudaStream_t; NULL = legacy default stream */
    int32_t tile_n;          /* T = LS sub-vector width = GEMM1 output-tile width:
                                0 = default (64 for the recomposed 16-bit path, block-sparse
                                layouts and the fp32 path; 128 for the unfused baseline and
                                SR_DECOMPOSE), or 64 / 128 */
    int32_t flags;           /* 0 = run the whole chain.  Otherwise an OR of SR_RUN_* stage bits:
                                only those kernels are launched, consuming the intermediates an
                                earlier call with the same arguments left in the workspace (used by
                                bench.py to time each kernel with events on the stream). */
} sr_exec;

/* Stage bits for sr_exec.flags. */
#define SR_RUN_GEMM1 1   /* GEMM1 + LS (recomposed) / GEMM1 writing scores (unfused) */
#define SR_RUN_REDUCE 2  /* IR kernel (SR_IR_KERNEL variant) / row softmax (unfused); no-op otherwise */
#define SR_RUN_GEMM2 4   /* GS + GEMM2 (recomposed) / GEMM2 on P (unfused) */
/* Variant bits for sr_exec.flags (recomposed 16-bit path; at most one).  Same results up to
 * rounding.  Default (none): the IR sub-layer merged inside GEMM1 (header comment).
 * SR_FUSE_IR: fold the IR sub-layer into GEMM2 instead (one warp of each GEMM2 CTA reduces the
 * item's m', d' before its GS warps need them; r' is formed on the fly and never written).
 * SURVEY.md NEXT-2. */
#define SR_FUSE_IR 16
/* Variant bit: SD, the softmax decomposition WITHOUT fusion ("SD" of Fig. 8):
 * plain GEMM1 (writes S) -> standalone LS (S -> X', m', d') -> IR -> standalone GS (X', r' -> Y)
 * -> plain GEMM2 (reads Y).  Six attention-matrix passes; the paper's intermediate ladder step
 * between the unfused baseline and SDF.  Workspace: sr_workspace_bytes with
 * fused = 2. */
#define SR_DECOMPOSE 32
/* Variant bit: the paper's three-kernel layout: GEMM1 + LS writes m', d';
 * a standalone IR kernel reduces them per row and writes r'_k = e^{m'_k - m} / d; GS + GEMM2
 * streams r' beside X'.  The only mode that writes d' and r' to the workspace. */
#define SR_IR_KERNEL 64
/* The whole recomposed chain in ONE launch -- the DEFAULT of the 16-bit
 * recomposed path (flags without a variant bit, tile_n 0 or 64): each persistent CTA runs GEMM1 +
 * LS + IR over its row-blocks, then GS + GEMM2 over the same rows after a CTA barrier (a CTA owns
 * whole rows, so no other CTA's results are needed).  X' still goes to the workspace and is read
 * back.  T = 64; stage bits are ignored (one kernel).  SR_ONE_KERNEL requests it explicitly. */
#define SR_ONE_KERNEL 128
/* Variant bit: the two-kernel chain GEMM1 + LS + IR -> GS + GEMM2 (the default before the
 * one-launch kernel; also what tile_n = 128 without a variant bit runs). */
#define SR_TWO_KERNELS 256
/* Modifier of the one-launch kernel (fp16): apply Global Scaling in GEMM2's prologue (Y = X' r'
 * rounded to fp16, then Y V) instead of accumulator-side (O += r'_k (X'_k V_k) in fp32, the
 * fp16 default).  bf16 always uses the prologue form. */
#define SR_GS_PROLOGUE 512
/* Modifier: skip the schedule upload.  The caller asserts that the workspace's schedule region
 * still holds what an earlier call with identical arguments (shape, mask content, causal, tile_n,
 * dtypes, variant and stage bits aside) wrote there, and that nothing has written it since (used by
 * bench.py to time single kernels with SR_RUN_* stage bits).  Wrong use reads a stale schedule. */
#define SR_SCHED_RESIDENT 1024
/* Variant bit: key-range split of long rows (the paper's three-kernel layout with chunked items):
 * GEMM1 + LS over chunks of <= L key tiles of a row-block (L = max(4, tiles / 296), about two chunks
 * per SM of a B200, so a layer with few long rows -- e.g. one GPU's share of a head-sharded layer --
 * still spreads over every SM), the standalone IR kernel over whole rows (writes r'), GS + GEMM2 over
 * the chunks -- each chunk of a split row-block writes an fp32 partial context, already scaled by the
 * global r' of its tiles -- and a combine kernel summing the partials in chunk order into out.
 * Workspace: SR_WS_RECOMPOSED (it reserves the partial region, off_partial). */
#define SR_SPLIT_KV 2048
/* Variant bit: GEMM1 + LS + IR and GS + GEMM2 run CONCURRENTLY in one persistent CTA per SM
 * (k_conc.cu): disjoint warps, shared memory and TMEM; GEMM2 takes each item (head,
 * 128-row block) over as soon as GEMM1 has stored its X' tiles, m' and row statistics, so the two
 * GEMMs overlap and X' is read back while it is still in L2 (it is still written to the workspace,
 * PAPER.md L171-L173).  16-bit inputs, D = 128, T = 64; same workspace as the default. */
#define SR_CONCURRENT 4096

/* Entry points (north star).  Returns SR_OK after enqueueing the kernels on ex->stream. */
sr_status sr_mha_dense(const void* q, const void* k, const void* v, void* out, int B, int H, int S,
                       int D, float scale, const sr_dense_mask* mask_or_null, int causal,
                       const sr_exec* ex);
sr_status sr_mha_blocksparse(const void* q, const void* k, const void* v, void* out, int B, int H,
                             int S, int D, float scale, const sr_block_layout* layout, int causal,
                             const sr_exec* ex);
sr_status sr_mha_sliding_window(const void* q, const void* k, const void* v, void* out, int B,
                                int H, int S, int D, float scale, const sr_window* win, int causal,
                                const sr_exec* ex);

/* In-repo traffic baseline: GEMM1 (scale+mask, writes scores) -> row softmax (reads scores,
 * writes P) -> GEMM2 (reads P).  Identical signatures and semantics; 16-bit dtypes only. */
sr_status sr_mha_dense_unfused(const void* q, const void* k, const void* v, void* out, int B,
                               int H, int S, int D, float scale, const sr_dense_mask* mask_or_null,
                               int causal, const sr_exec* ex);
sr_status sr_mha_blocksparse_unfused(const void* q, const void* k, const void* v, void* out, int B,
                                     int H, int S, int D, float scale,
                                     const sr_block_layout* layout, int causal, const sr_exec* ex);
sr_status sr_mha_sliding_window_unfused(const void* q, const void* k, const void* v, void* out,
                                        int B, int H, int S, int D, float scale,
                                        const sr_window* win, int causal, const sr_exec* ex);

/* Training backward (Sec. 6).  Given the upstream gradient
 * dout = dE/dO, computes dq = dE/dQ, dk = dE/dK, dv = dE/dV of the same layer, using only what the
 * forward left in the workspace -- the unnormalised X' tiles, m' and the per-row statistics --
 * never the softmax input x (the paper's argument: Eq. (3) expresses dE/dx through y alone):
 *
 *   P    = X' * r'_k,  r'_k = e^{m'_k - m} / d          (Global Scaling, recomputed per tile)
 *   dP   = dO V^T                                         (tensor cores, dE/dy)
 *   dS'  = scale * P (dP - delta),  delta_i = sum_d dO_id O_id      (Eq. 3 row form: dE/dx_k =
 *          y_k (dE/dy_k - sum_i dE/dy_i y_i), and sum_j P_ij dP_ij = dO_i . O_i)
 *   dq   = dS' K (accumulated in the dS' kernel),  dk = dS'^T Q,  dv = P^T dO   (tensor cores)
 *
 * Contract: the call must follow a forward call of the SAME entry point with the same q, k, v,
 * shape, mask / layout, causal, tile_n, in_dtype and out_dtype, in the default mode (flags 0: the
 * IR merged in GEMM1 -- the only mode that leaves per-row statistics), on the same workspace,
 * sized with sr_workspace_bytes(entry, SR_WS_TRAIN, ...).  `out` is that forward's output
 * (out_dtype).  dout: DEVICE, [B][H][S][D], in_dtype.  dq, dk, dv: DEVICE, [B][H][S][D],
 * out_dtype, fully overwritten, must not overlap q, k, v, out, dout or each other.  16-bit
 * in_dtype only (SR_ERR_UNSUPPORTED for F32).  ex->flags: 0, or SR_RUN_GEMM1 (row statistics +
 * dS' + dq kernels), SR_RUN_GEMM2 (dk and dv kernel) for per-kernel timing (SR_RUN_REDUCE: the
 * separate dq kernel of SR_BWD_DQ_SEPARATE=1 runs only).  Three launches (row statistics, dS' + dq,
 * dk + dv), stream-ordered, asynchronous; errors as for the forward. */
sr_status sr_mha_dense_bwd(const void* q, const void* k, const void* v, const void* out, const void* dout,
                           void* dq, void* dk, void* dv, int B, int H, int S, int D, float scale,
                           const sr_dense_mask* mask_or_null, int causal, const sr_exec* ex);
sr_status sr_mha_blocksparse_bwd(const void* q, const void* k, const void* v, const void* out,
                                 const void* dout, void* dq, void* dk, void* dv, int B, int H, int S,
                                 int D, float scale, const sr_block_layout* layout, int causal,
                                 const sr_exec* ex);
sr_status sr_mha_sliding_window_bwd(const void* q, const void* k, const void* v, const void* out,
                                    const void* dout, void* dq, void* dk, void* dv, int B, int H,
                                    int S, int D, float scale, const sr_window* win, int causal,
                                    const sr_exec* ex);

/* Workspace modes for sr_workspace_bytes / sr_workspace_query (the `fused` argument). */
#define SR_WS_UNFUSED 0
#define SR_WS_RECOMPOSED 1
#define SR_WS_SD 2
#define SR_WS_TRAIN 3 /* recomposed forward + backward: adds the dS' tiles and bstat */

/* Which entry point a workspace query is for. */
typedef enum { SR_E_DENSE = 0, SR_E_BLOCKSPARSE = 1, SR_E_WINDOW = 2 } sr_entry;

/* Workspace layout (all offsets in bytes from ex->workspace; 256-byte aligned):
 *   A tile is 128 query rows x T keys.  Every (head, row-block, listed key tile) owns a "slot";
 *   slot s of head g has global id  g * slots_per_head + s.
 *   xprime   recomposed: X' tiles, unfused: the score tiles S and then P (2 regions), each tile
 *            128*T elements of xprime_elt_bytes; 16-bit tiles are stored in the canonical
 *            SWIZZLE_128B K-major layout [T/64][128 rows][64 cols] with the 16-byte chunk index
 *            XOR (row & 7); fp32 tiles are plain row-major [128][T].
 *   mprime, dprime, rprime   fp32 [slot id][128 rows]  (m' in natural-log units)
 *   rowstat  fp32 [2][2][B*H*S] (default mode): two partial row statistics per query row, each
 *            m_w (natural-log units) then d_w; the row's m = max_w m_w, d = sum_w e^{m_w - m} d_w
 *   ds, bstat  SR_WS_TRAIN only (backward): dS' tiles; per-row m, 1/d, delta.  The backward also
 *            writes r' (rprime) for every listed tile.
 *   sched    the call's tile schedule (int32 words: tile lists, item descriptors, per-CTA ranges),
 *            written by each call before its kernels run; sched_bytes reserves room for any SM count
 */
typedef struct {
    int32_t tile_n;           /* T actually used */
    int32_t slots_per_head;
    int64_t n_slots;          /* B*H*slots_per_head */
    int32_t xprime_elt_bytes; /* 2 (16-bit paths) or 4 (fp32 path) */
    size_t off_xprime, off_mprime, off_dprime, off_rprime, off_p;  /* off_p: unfused P region */
    size_t off_rowstat;       /* recomposed: per-row partial (m, d) of the default (IR in GEMM1) mode */
    size_t total_bytes;
    size_t off_ds;            /* SR_WS_TRAIN: dS' tiles, same slots / layout as X', in_dtype */
    size_t off_bstat;         /* SR_WS_TRAIN: fp32 [3][B*H*S]: m, 1/d, delta per query row */
    size_t off_sched;         /* tile schedule region (every mode) */
    size_t sched_bytes;
    size_t off_partial;       /* SR_WS_RECOMPOSED: fp32 [slot][128][D] partial contexts of SR_SPLIT_KV */
} sr_ws_info;

/* Workspace bytes needed by an entry point; `mask_or_layout` is the same pointer passed to it
 * (sr_dense_mask*, sr_block_layout* or sr_window*; may be NULL for dense).  fused: 1 recomposed
 * (also SR_FUSE_IR), 0 unfused, 2 SD (SR_DECOMPOSE), 3 training forward + backward (SR_WS_TRAIN).  Returns 0 on invalid/unsupported arguments
 * (see sr_last_error()). */
size_t sr_workspace_bytes(sr_entry entry, int fused, int B, int H, int S, int D, sr_dtype in_dtype,
                          const void* mask_or_layout, int causal, int tile_n);
/* Same, with the full layout of the workspace (for tests that read X', m', d', r' back). */
sr_status sr_workspace_query(sr_entry entry, int fused, int B, int H, int S, int D,
                             sr_dtype in_dtype, const void* mask_or_layout, int causal, int tile_n,
                             sr_ws_info* info);

/* Host-side tile schedule of a call, for tests and the byte model: number of stored score
 * elements (tiles x 128 x T, counting only valid 64-row halves) and tile count. */
sr_status sr_schedule_stats(sr_entry entry, int B, int H, int S, const void* mask_or_layout,
                            int causal, int tile_n, int64_t* n_tiles, int64_t* stored_elems);

const char* sr_status_string(sr_status s);
const char* sr_last_error(void);
/* Kernel launches issued by the calling thread since the library was loaded (for bench.py's
 * gpu_launches count). */
int64_t sr_launch_count(void);
const char* sr_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SR_MHA_H */
