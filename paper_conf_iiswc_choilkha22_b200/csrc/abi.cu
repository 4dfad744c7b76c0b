// abi.cu -- the C ABI of include/sr_mha.h: argument validation, tile schedules, workspace
// layout, schedule cache, dispatch to the kernels.  Host code only.
//
// The tile schedule is the B200 form of the paper's TB work distribution (PAPER.md L112, L135,
// Fig. 3-4): GEMM1 and GEMM2 iterate "items" (head, 128-row block) and, per item, the list of key
// tiles that hold at least one kept element.  Fully masked tiles (causal upper triangle, padded
// keys, absent sparse blocks, far-off band) are never computed, stored or read (reading R18).
#include <algorithm>
#include <array>
#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <list>
#include <map>
#include <memory>
#include <mutex>
#include <queue>
#include <string>
#include <unordered_map>
#include <vector>

#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: ranges show up in nsys / ncu --nvtx when a tool is attached

#include "../../include/sr_mha.h"
#include "sr_internal.h"

using namespace sr;

namespace {

thread_local char g_err[512] = "";
std::atomic<int64_t> g_launches{0};

sr_status fail(sr_status s, const char* fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return s;
}

int dtype_bytes(int dt) { return dt == SR_F32 ? 4 : 2; }

// ------------------------------------------------------------------------------ schedules

struct HostSched {
    int T = 0, H = 1, n_rb = 0, n_lh = 1, lh_mode = LH_ONE;
    std::vector<int32_t> tp, tinfo, items, kv_len;
    std::vector<int32_t> cta_ptr;  // device schedules only: items grouped per persistent CTA
    // GEMM1 pair schedule: row-blocks 2j, 2j+1 of a head share every K tile of the union of their
    // lists.  pp [n_lh][n_pair+1] offsets into pent; pent 4 ints per union entry
    // {kt | half bits of 2j << 16 | half bits of 2j+1 << 18, tinfo index in 2j's list or -1, same
    // for 2j+1, 0}; pitems g * n_pair + j grouped per CTA (pcta_ptr).
    int n_pair = 0;
    std::vector<int32_t> pp, pent, pitems, pcta_ptr;
    double pair_saving = 0.0;  // 1 - (pair union entries / listed tiles): the K-tile loads pairs save
    // column schedule (training backward, dK / dV): cpp [n_lh][n_cb+1] offsets into cent (4 ints
    // per entry, see DevSched::cent); citems g * n_cb + c grouped per CTA (ccta_ptr)
    int n_cb = 0;
    std::vector<int32_t> cpp, cent, citems, ccta_ptr;
    // unfused softmax: the 64-row halves whose rows hold more than kSmShortChunks 64-key chunks
    // ((g * n_rb + rb) * 2 + half), run by their own launch with their rows spread over CTAs
    std::vector<int32_t> sm_long;
    int slots_per_head = 0;
    int max_rb_tiles = 0;
    // key-range split plan (SR_SPLIT_KV): every item as chunks of <= split_L tiles, 4 ints each
    // {item, t0, t1, partial slot or -1}; comb 4 ints per split row-block {item, slot0, chunks, 0}
    int split_L = 0;
    std::vector<int32_t> chunks, comb;
    int64_t n_partial = 0;
    int64_t n_tiles = 0;       // over all B*H heads
    int64_t stored_elems = 0;  // valid 64-row halves x 64 x T, over all heads
};

struct Request {
    sr_entry entry;
    int B, H, S, causal, T;
    const int32_t* kv_len = nullptr;
    const sr_block_layout* lay = nullptr;
    int window = 0, n_global = 0;
};

// Does the half-tile rows [r0, r1] x keys [c0, c1] hold a kept element of the window mask?
// (i, j) kept iff (|i-j| <= w2 or i < g or j < g) and (!causal or j <= i).
bool window_half_valid(int r0, int r1, int c0, int c1, int w2, int g, bool causal)
{
    // band: j - i in [-w2, causal ? 0 : w2]  intersect  [c0 - r1, c1 - r0]
    int hi = causal ? 0 : w2;
    if (c0 - r1 <= hi && c1 - r0 >= -w2) return true;
    // global rows i < g (with causal, needs some j <= i, best i = min(r1, g-1))
    if (r0 < g) {
        int imax = std::min(r1, g - 1);
        if (!causal || c0 <= imax) return true;
    }
    // global columns j < g (with causal, needs some i >= j, best j = c0)
    if (c0 < g) {
        if (!causal || r1 >= c0) return true;
    }
    return false;
}

sr_status build_sched(const Request& r, HostSched& hs)
{
    const int S = r.S, T = r.T;
    hs.T = T;
    hs.H = r.H;
    // S % 128 == 64: the last row-block's upper 64-row half lies beyond the head (never valid: its
    // tiles are neither computed into X' nor read, and every kernel skips writes of rows >= S)
    hs.n_rb = (S + kRowBlock - 1) / kRowBlock;
    const int nkt = S / T;
    std::vector<std::vector<std::pair<int, int>>> lists;  // per (lh, rb): (kt, half bits)
    if (r.entry == SR_E_DENSE || r.entry == SR_E_WINDOW) {
        hs.lh_mode = (r.entry == SR_E_DENSE && r.kv_len) ? LH_BATCH : LH_ONE;
        hs.n_lh = hs.lh_mode == LH_BATCH ? r.B : 1;
        for (int lh = 0; lh < hs.n_lh; ++lh) {
            int kvl = (hs.lh_mode == LH_BATCH) ? r.kv_len[lh] : S;
            for (int rb = 0; rb < hs.n_rb; ++rb) {
                std::vector<std::pair<int, int>> L;
                for (int kt = 0; kt < nkt; ++kt) {
                    int c0 = kt * T, c1 = c0 + T - 1, bits = 0;
                    for (int h = 0; h < 2; ++h) {
                        int r0 = rb * kRowBlock + h * kHalf, r1 = r0 + kHalf - 1;
                        bool ok;
                        if (r0 >= S)
                            ok = false;
                        else if (r.entry == SR_E_DENSE)
                            ok = c0 < kvl && (!r.causal || c0 <= r1);
                        else
                            ok = window_half_valid(r0, r1, c0, std::min(c1, S - 1), r.window / 2, r.n_global, r.causal);
                        if (ok) bits |= 1 << h;
                    }
                    if (bits) L.push_back({kt, bits});
                }
                lists.push_back(std::move(L));
            }
        }
    } else {  // block-sparse: pair the 64-row block-rows 2rb, 2rb+1 and take the union of columns
        const sr_block_layout* lay = r.lay;
        hs.lh_mode = lay->layout_heads == 1 ? LH_ONE : LH_HEAD;
        hs.n_lh = lay->layout_heads;
        const int nb = S / lay->block;
        for (int lh = 0; lh < hs.n_lh; ++lh) {
            const int32_t* rp = lay->row_ptr + (size_t)lh * (nb + 1);
            for (int rb = 0; rb < hs.n_rb; ++rb) {
                std::map<int, int> cols;
                for (int h = 0; h < 2; ++h) {
                    int br = 2 * rb + h;
                    if (br >= nb) continue;  // S % 128 == 64: no block-row beyond the head
                    for (int32_t t = rp[br]; t < rp[br + 1]; ++t) {
                        int c = lay->col_idx[t];
                        if (r.causal && c > br) continue;  // block entirely above the diagonal
                        cols[c] |= 1 << h;
                    }
                }
                std::vector<std::pair<int, int>> L(cols.begin(), cols.end());
                lists.push_back(std::move(L));
            }
        }
    }
    // flatten
    hs.tp.assign((size_t)hs.n_lh * (hs.n_rb + 1), 0);
    int32_t off = 0;
    std::vector<int64_t> lh_elems(hs.n_lh, 0), lh_tiles(hs.n_lh, 0);
    for (int lh = 0; lh < hs.n_lh; ++lh) {
        hs.tp[(size_t)lh * (hs.n_rb + 1)] = off;
        for (int rb = 0; rb < hs.n_rb; ++rb) {
            for (auto& kb : lists[(size_t)lh * hs.n_rb + rb]) {
                hs.tinfo.push_back(kb.first | (kb.second << 16));
                lh_elems[lh] += (int64_t)__builtin_popcount(kb.second) * kHalf * T;
                lh_tiles[lh] += 1;
            }
            hs.max_rb_tiles = std::max<int>(hs.max_rb_tiles, (int)hs.tinfo.size() - off);
            off = (int32_t)hs.tinfo.size();
            hs.tp[(size_t)lh * (hs.n_rb + 1) + rb + 1] = off;
        }
        hs.slots_per_head = std::max<int>(hs.slots_per_head, (int)lh_tiles[lh]);
    }
    // items, longest first (static LPT order; ties keep head-major order)
    const int BH = r.B * r.H;
    std::vector<std::pair<int, int32_t>> it;
    it.reserve((size_t)BH * hs.n_rb);
    for (int g = 0; g < BH; ++g) {
        int lh = hs.lh_mode == LH_ONE ? 0 : (hs.lh_mode == LH_BATCH ? g / r.H : g % r.H);
        hs.n_tiles += lh_tiles[lh];
        hs.stored_elems += lh_elems[lh];
        for (int rb = 0; rb < hs.n_rb; ++rb) {
            const int32_t* tp = &hs.tp[(size_t)lh * (hs.n_rb + 1)];
            it.push_back({tp[rb + 1] - tp[rb], g * hs.n_rb + rb});
        }
    }
    std::stable_sort(it.begin(), it.end(), [](auto& a, auto& b) { return a.first > b.first; });
    hs.items.resize(it.size());
    for (size_t i = 0; i < it.size(); ++i) hs.items[i] = it[i].second;
    if (r.kv_len) hs.kv_len.assign(r.kv_len, r.kv_len + r.B);
    // long softmax halves (global rows of BigBird / Longformer, dense rows), listed only for layers
    // whose longest rows take the softmax's two-launch path (> 4 x 8 chunks, k_softmax.cu)
    for (int g = 0; hs.max_rb_tiles * (T / 64) > 32 && g < BH; ++g) {
        const int lh = hs.lh_mode == LH_ONE ? 0 : (hs.lh_mode == LH_BATCH ? g / r.H : g % r.H);
        const int32_t* tp = &hs.tp[(size_t)lh * (hs.n_rb + 1)];
        for (int rb = 0; rb < hs.n_rb; ++rb)
            for (int h = 0; h < 2; ++h) {
                int n = 0;
                for (int t = tp[rb]; t < tp[rb + 1]; ++t) n += (tinfo_half(hs.tinfo[t]) >> h) & 1;
                if (n * (T / 64) > kSmShortChunks) hs.sm_long.push_back((g * hs.n_rb + rb) * 2 + h);
            }
    }
    // pair lists: merge the (kt-ascending) lists of row-blocks 2j and 2j+1
    hs.n_pair = (hs.n_rb + 1) / 2;
    hs.pp.assign((size_t)hs.n_lh * (hs.n_pair + 1), 0);
    for (int lh = 0; lh < hs.n_lh; ++lh) {
        const int32_t* tp = &hs.tp[(size_t)lh * (hs.n_rb + 1)];
        hs.pp[(size_t)lh * (hs.n_pair + 1)] = (int32_t)(hs.pent.size() / 4);
        for (int j = 0; j < hs.n_pair; ++j) {
            int ia = tp[2 * j], ea = tp[2 * j + 1];
            int ib = 2 * j + 1 < hs.n_rb ? tp[2 * j + 1] : 0, eb = 2 * j + 1 < hs.n_rb ? tp[2 * j + 2] : 0;
            while (ia < ea || ib < eb) {
                const int ka = ia < ea ? tinfo_kt(hs.tinfo[ia]) : INT32_MAX;
                const int kb = ib < eb ? tinfo_kt(hs.tinfo[ib]) : INT32_MAX;
                const int kt = std::min(ka, kb);
                int32_t w = kt, ta = -1, tb = -1;
                if (ka == kt) { w |= tinfo_half(hs.tinfo[ia]) << 16; ta = ia++; }
                if (kb == kt) { w |= tinfo_half(hs.tinfo[ib]) << 18; tb = ib++; }
                hs.pent.insert(hs.pent.end(), {w, ta, tb, 0});
            }
            hs.pp[(size_t)lh * (hs.n_pair + 1) + j + 1] = (int32_t)(hs.pent.size() / 4);
        }
    }
    for (int g = 0; g < BH; ++g)
        for (int j = 0; j < hs.n_pair; ++j) hs.pitems.push_back(g * hs.n_pair + j);
    if (!hs.tinfo.empty()) hs.pair_saving = 1.0 - (double)(hs.pent.size() / 4) / (double)hs.tinfo.size();
    // column lists (the transpose of the row lists, for dK = dS'^T Q and dV = P^T dO): per 128-key
    // column block, the row-blocks that list one of its key tiles, ascending
    hs.n_cb = (S + kRowBlock - 1) / kRowBlock;
    const int per = kRowBlock / T;  // key tiles per column block
    hs.cpp.assign((size_t)hs.n_lh * (hs.n_cb + 1), 0);
    for (int lh = 0; lh < hs.n_lh; ++lh) {
        const int32_t* tp = &hs.tp[(size_t)lh * (hs.n_rb + 1)];
        std::vector<std::vector<std::array<int32_t, 4>>> cols(hs.n_cb);
        for (int rb = 0; rb < hs.n_rb; ++rb)
            for (int t = tp[rb]; t < tp[rb + 1]; ++t) {
                const int kt = tinfo_kt(hs.tinfo[t]), c = kt / per, u = kt % per;
                auto& L = cols[c];
                if (L.empty() || (L.back()[0] & 0xFFFF) != rb) L.push_back({rb, -1, -1, 0});
                L.back()[0] |= tinfo_half(hs.tinfo[t]) << (16 + 2 * u);
                L.back()[1 + u] = t;
            }
        hs.cpp[(size_t)lh * (hs.n_cb + 1)] = (int32_t)(hs.cent.size() / 4);
        for (int c = 0; c < hs.n_cb; ++c) {
            for (auto& e : cols[c]) hs.cent.insert(hs.cent.end(), e.begin(), e.end());
            hs.cpp[(size_t)lh * (hs.n_cb + 1) + c + 1] = (int32_t)(hs.cent.size() / 4);
        }
    }
    for (int g = 0; g < BH; ++g)
        for (int c = 0; c < hs.n_cb; ++c) hs.citems.push_back(g * hs.n_cb + c);
    // key-range split: rows whose tile list exceeds L = max(4, tiles / (2 x 148)) -- a chunk count of
    // about two per SM of a B200 -- are cut into near-equal chunks (device-independent, so the
    // workspace size is known on the host)
    hs.split_L = (int)std::max<int64_t>(4, (hs.n_tiles + 2 * kSplitRefSms - 1) / (2 * kSplitRefSms));
    for (int g = 0; g < BH; ++g) {
        const int lh = hs.lh_mode == LH_ONE ? 0 : (hs.lh_mode == LH_BATCH ? g / r.H : g % r.H);
        const int32_t* tp = &hs.tp[(size_t)lh * (hs.n_rb + 1)];
        for (int rb = 0; rb < hs.n_rb; ++rb) {
            const int w = g * hs.n_rb + rb, t0 = tp[rb], n = tp[rb + 1] - tp[rb];
            const int nc = n > hs.split_L ? (n + hs.split_L - 1) / hs.split_L : 1;
            for (int c = 0; c < nc; ++c) {
                const int a = t0 + (int)((int64_t)n * c / nc), b = t0 + (int)((int64_t)n * (c + 1) / nc);
                hs.chunks.insert(hs.chunks.end(), {w, a, b, nc > 1 ? (int32_t)(hs.n_partial + c) : -1});
            }
            if (nc > 1) {
                hs.comb.insert(hs.comb.end(), {w, (int32_t)hs.n_partial, nc, 0});
                hs.n_partial += nc;
            }
        }
    }
    return SR_OK;
}

// ------------------------------------------------------------------------------ validation

int default_T(sr_entry e, int in_dtype, int mode)
{
    if (in_dtype == SR_F32) return 64;
    // the recomposed 16-bit default (and training) is the one-launch kernel (k_fused.cu), whose
    // SPLIT GEMM1 epilogue runs T = 64 sub-vectors in 128-key macro tiles
    if (mode == 1 || mode == 3) return 64;
    // T = the GEMM1 output-tile width: 128 on the tensor cores; block-sparse
    // layouts fix the sub-vector to the 64-key block (two of them share one 128-key MMA tile)
    return e == SR_E_BLOCKSPARSE ? 64 : 128;
}

sr_status check_request(sr_entry e, int B, int H, int S, int D, int in_dtype,
                        const void* mask_or_layout, int causal, int tile_n, Request& r, int mode)
{
    if (B <= 0 || H <= 0 || S <= 0 || D <= 0)
        return fail(SR_ERR_INVALID, "B, H, S, D must be positive (got %d %d %d %d)", B, H, S, D);
    if (in_dtype != SR_F32 && in_dtype != SR_F16 && in_dtype != SR_BF16)
        return fail(SR_ERR_INVALID, "unknown in_dtype %d", in_dtype);
    if (S % kHalf != 0) return fail(SR_ERR_UNSUPPORTED, "S=%d must be a multiple of 64", S);
    if (S > 65536 * 64) return fail(SR_ERR_UNSUPPORTED, "S=%d too large", S);
    if (D != 64 && D != 128) return fail(SR_ERR_UNSUPPORTED, "D=%d must be 64 or 128", D);
    if ((int64_t)B * H * ((S + kRowBlock - 1) / kRowBlock) > INT32_MAX / 2)
        return fail(SR_ERR_UNSUPPORTED, "too many (head, row-block) items");
    if (tile_n != 0 && tile_n != 64 && tile_n != 128)
        return fail(SR_ERR_UNSUPPORTED, "tile_n=%d must be 0, 64 or 128", tile_n);
    int T = tile_n ? tile_n : default_T(e, in_dtype, mode);
    if (T == 128 && S % 128 != 0) {  // 128-key sub-vectors need S % 128 == 0; the default falls back to 64
        if (tile_n) return fail(SR_ERR_UNSUPPORTED, "tile_n=128 needs S %% 128 == 0 (S=%d)", S);
        T = 64;
    }
    if (in_dtype == SR_F32 && T != 64) return fail(SR_ERR_UNSUPPORTED, "fp32 path uses T=64");
    r = Request{e, B, H, S, causal ? 1 : 0, T};
    if (e == SR_E_DENSE) {
        const sr_dense_mask* m = (const sr_dense_mask*)mask_or_layout;
        if (m && m->kv_len) {
            for (int b = 0; b < B; ++b)
                if (m->kv_len[b] < 0 || m->kv_len[b] > S)
                    return fail(SR_ERR_INVALID, "kv_len[%d]=%d outside [0, S=%d]", b, m->kv_len[b], S);
            r.kv_len = m->kv_len;
        }
    } else if (e == SR_E_BLOCKSPARSE) {
        const sr_block_layout* l = (const sr_block_layout*)mask_or_layout;
        if (!l || !l->row_ptr || !l->col_idx) return fail(SR_ERR_INVALID, "block layout missing");
        if (l->block != 64) return fail(SR_ERR_UNSUPPORTED, "block=%d must be 64", l->block);
        if (l->layout_heads != 1 && l->layout_heads != H)
            return fail(SR_ERR_INVALID, "layout_heads=%d must be 1 or H=%d", l->layout_heads, H);
        if (T != 64) return fail(SR_ERR_UNSUPPORTED, "block-sparse uses T = block = 64");
        int nb = S / 64;
        for (int h = 0; h < l->layout_heads; ++h) {
            const int32_t* rp = l->row_ptr + (size_t)h * (nb + 1);
            if (rp[0] < 0) return fail(SR_ERR_INVALID, "row_ptr[%d][0] < 0", h);
            for (int rr = 0; rr < nb; ++rr) {
                if (rp[rr + 1] < rp[rr]) return fail(SR_ERR_INVALID, "row_ptr decreasing (head %d row %d)", h, rr);
                for (int32_t t = rp[rr]; t < rp[rr + 1]; ++t) {
                    int c = l->col_idx[t];
                    if (c < 0 || c >= nb) return fail(SR_ERR_INVALID, "col_idx %d out of range (head %d row %d)", c, h, rr);
                    if (t > rp[rr] && c <= l->col_idx[t - 1])
                        return fail(SR_ERR_INVALID, "col_idx not strictly ascending (head %d row %d)", h, rr);
                }
            }
        }
        r.lay = l;
    } else if (e == SR_E_WINDOW) {
        const sr_window* w = (const sr_window*)mask_or_layout;
        if (!w) return fail(SR_ERR_INVALID, "window descriptor missing");
        if (w->window < 0 || w->n_global < 0 || w->n_global > S)
            return fail(SR_ERR_INVALID, "bad window=%d / n_global=%d", w->window, w->n_global);
        r.window = w->window;
        r.n_global = w->n_global;
    } else {
        return fail(SR_ERR_INVALID, "unknown entry %d", (int)e);
    }
    return SR_OK;
}

// ------------------------------------------------------------------------------ cache
//
// Host schedules are cached by mask content in a bounded LRU (host memory only: nothing on the
// device is library-owned).  The device form of a schedule is a word blob that every call uploads
// into its own workspace (k_sched.cu), so a cache eviction can never invalidate a pending launch or
// a captured graph.

// Word groups of the blob, each a contiguous, 16-B aligned range; a call uploads only the groups
// its kernels read.
enum BlobGroup { G_BASE = 0, G_ITEMS, G_PAIR, G_FP, G_COL, G_SML, G_N };
constexpr int kMaxCta = 1024;  // bound on persistent CTAs per launch (the workspace reserves it)

struct BlobLayout {  // int32-word offsets inside the blob
    size_t tp, tinfo, kv, desc, items, cta, iri, psl, comb, pdesc, pent, pcta, fp, fpcta, cdesc, cent, ccta, slong;
    size_t g_off[G_N], g_len[G_N];
    size_t words;
};

struct DevBlob {
    int n_sm = 0;
    bool split = false;
    double imbalance = 1.0;  // LPT: most loaded CTA / mean load over n_sm SMs (row-block items)
    std::vector<int32_t> w;
    BlobLayout L{};
    DevSched rel{};  // scalar fields of the device schedule (pointers filled per call)
};

struct CachedSched {
    HostSched hs;
    std::mutex mu;                              // guards blobs
    std::vector<std::shared_ptr<DevBlob>> blobs;  // one per SM count seen (normally one)
};

std::mutex g_mu;
constexpr size_t kCacheCap = 128;
std::list<std::string> g_lru;  // most recent first
std::unordered_map<std::string, std::pair<std::shared_ptr<CachedSched>, std::list<std::string>::iterator>> g_cache;

std::string sched_key(const Request& r)
{
    std::string k;
    auto put = [&](int64_t x) { k.append((const char*)&x, sizeof(x)); };
    put(r.entry); put(r.B); put(r.H); put(r.S); put(r.causal); put(r.T);
    put(r.window); put(r.n_global);
    if (r.kv_len) { put(1); for (int b = 0; b < r.B; ++b) put(r.kv_len[b]); } else put(0);
    if (r.lay) {
        int nb = r.S / 64;
        put(r.lay->layout_heads);
        for (int h = 0; h < r.lay->layout_heads; ++h) {
            const int32_t* rp = r.lay->row_ptr + (size_t)h * (nb + 1);
            for (int i = 0; i <= nb; ++i) put(rp[i] - rp[0]);
            k.append((const char*)(r.lay->col_idx + rp[0]), sizeof(int32_t) * (rp[nb] - rp[0]));
        }
    }
    return k;
}

// Word layout of the blob for given per-CTA-range lengths (n_cta + 1 entries each).  The workspace
// region is sized with kMaxCta so it fits every device.
BlobLayout blob_layout(const HostSched& h, size_t n_desc, size_t n_cta_ptr, size_t n_pcta_ptr, size_t n_ccta_ptr)
{
    BlobLayout L{};
    size_t o = 0;
    auto pad = [&] { o = (o + 3) / 4 * 4; };
    auto grp = [&](int g, size_t start) { L.g_off[g] = start; pad(); L.g_len[g] = o - start; };
    size_t s = o;  // G_BASE: tp, tinfo, kv_len
    L.tp = o; o += h.tp.size();
    L.tinfo = o; o += std::max<size_t>(h.tinfo.size(), 1);
    L.kv = o; o += h.kv_len.size();
    grp(G_BASE, s);
    s = o;  // G_ITEMS: item descriptors (16-B aligned), items, cta_ptr
    L.desc = o; o += 4 * n_desc;    // row-blocks, or their chunks with SR_SPLIT_KV
    L.items = o; o += h.items.size();
    L.cta = o; o += n_cta_ptr;
    L.psl = o; o += n_desc;          // SR_SPLIT_KV: partial slot of each descriptor
    pad();                           // int4 records below
    L.comb = o; o += std::max<size_t>(h.comb.size(), 4);
    L.iri = o; o += 4 * h.items.size();  // the standalone IR kernel's row-blocks (longest first), as descriptors
    grp(G_ITEMS, s);
    s = o;  // G_PAIR: pair descriptors, union entries, pcta_ptr
    L.pdesc = o; o += 4 * h.pitems.size();
    L.pent = o; o += std::max<size_t>(h.pent.size(), 4);
    L.pcta = o; o += n_pcta_ptr;
    grp(G_PAIR, s);
    s = o;  // G_FP: the pair assignment unrolled into row-block descriptors, fpcta_ptr
    L.fp = o; o += 4 * h.items.size();
    L.fpcta = o; o += n_pcta_ptr;
    grp(G_FP, s);
    s = o;  // G_COL: column descriptors, column entries, ccta_ptr
    L.cdesc = o; o += 4 * h.citems.size();
    L.cent = o; o += std::max<size_t>(h.cent.size(), 4);
    L.ccta = o; o += n_ccta_ptr;
    grp(G_COL, s);
    s = o;  // G_SML: the unfused softmax's long-row halves (uploaded by the unfused path only)
    L.slong = o; o += std::max<size_t>(h.sm_long.size(), 1);
    grp(G_SML, s);
    L.words = o;
    return L;
}

size_t sched_region_bytes(const HostSched& h)
{
    return blob_layout(h, std::max(h.items.size(), h.chunks.size() / 4), kMaxCta + 1, kMaxCta + 1, kMaxCta + 1).words *
           sizeof(int32_t);
}

void lpt_assign(HostSched& h, int n_cta);

// The device blob of a schedule for n_sm persistent CTAs (built once, then shared read-only).
int64_t lpt_item_cost();
void lpt_assign(std::vector<int32_t>& items, const std::vector<int64_t>& cost, int n_cta, std::vector<int32_t>& cta_ptr);

std::shared_ptr<DevBlob> make_blob(const HostSched& h0, int n_sm, bool split)
{
    HostSched h = h0;  // the LPT pass reorders items: keep the cached host schedule device-neutral
    lpt_assign(h, std::min(n_sm, kMaxCta));
    auto db = std::make_shared<DevBlob>();
    db->n_sm = n_sm;
    db->split = split;
    auto lh_of_g = [&](int g) { return h.lh_mode == LH_ONE ? 0 : (h.lh_mode == LH_BATCH ? g / h.H : g % h.H); };
    // item descriptors {item, t0, t1, tp[lh][0]} grouped per CTA, and each one's partial slot: the
    // LPT assignment of row-blocks, or (SR_SPLIT_KV) of the chunks of the split plan
    std::vector<int32_t> desc, psl, cta_ptr;
    if (!split) {
        for (int32_t it : h.items) {
            const int g = it / h.n_rb, rb = it % h.n_rb;
            const int32_t* tp = &h.tp[(size_t)lh_of_g(g) * (h.n_rb + 1)];
            desc.insert(desc.end(), {it, tp[rb], tp[rb + 1], tp[0]});
            psl.push_back(-1);
        }
        cta_ptr = h.cta_ptr;
        double tot = 0.0, mx = 0.0;  // how far the longest items stick out of a balanced share
        for (size_t c = 0; c + 1 < cta_ptr.size(); ++c) {
            double ld = 0.0;
            for (int i = cta_ptr[c]; i < cta_ptr[c + 1]; ++i)
                ld += 2.0 * (desc[4 * i + 2] - desc[4 * i + 1]) + (double)lpt_item_cost();
            tot += ld;
            mx = std::max(mx, ld);
        }
        db->imbalance = tot > 0.0 ? mx / (tot / std::max(n_sm, 1)) : 1.0;
    } else {
        const size_t nch = h.chunks.size() / 4;
        std::vector<int32_t> order(nch);
        std::vector<int64_t> cost(nch);
        for (size_t i = 0; i < nch; ++i) {
            order[i] = (int32_t)i;
            cost[i] = 2 * (int64_t)(h.chunks[4 * i + 2] - h.chunks[4 * i + 1]) + lpt_item_cost();
        }
        lpt_assign(order, cost, std::min(n_sm, kMaxCta), cta_ptr);
        for (int32_t i : order) {
            const int32_t* c = &h.chunks[4 * (size_t)i];
            const int g = c[0] / h.n_rb;
            desc.insert(desc.end(), {c[0], c[1], c[2], h.tp[(size_t)lh_of_g(g) * (h.n_rb + 1)]});
            psl.push_back(c[3]);
        }
    }
    BlobLayout L = blob_layout(h, desc.size() / 4, cta_ptr.size(), h.pcta_ptr.size(), h.ccta_ptr.size());
    db->L = L;
    std::vector<int32_t>& w = db->w;
    w.assign(L.words, 0);
    auto put = [&](size_t off, const std::vector<int32_t>& v) { std::copy(v.begin(), v.end(), w.begin() + off); };
    put(L.tp, h.tp);
    put(L.tinfo, h.tinfo);
    put(L.kv, h.kv_len);
    put(L.desc, desc);
    put(L.items, h.items);
    put(L.cta, cta_ptr);
    size_t o;
    o = L.iri;  // the IR kernel's row-block descriptors {first slot, tiles, first tile, item}, before the
                // LPT pass (longest first); the slot is g * slots_per_head + t0 - tp[lh][0] (no division on the device)
    for (int32_t it : h0.items) {
        const int g = it / h0.n_rb, rb = it % h0.n_rb;
        const int32_t* tp = &h0.tp[(size_t)(h0.lh_mode == LH_ONE ? 0 : (h0.lh_mode == LH_BATCH ? g / h0.H : g % h0.H)) *
                                   (h0.n_rb + 1)];
        const int32_t dd[4] = {(int32_t)((int64_t)g * h0.slots_per_head + tp[rb] - tp[0]), tp[rb + 1] - tp[rb], tp[rb], it};
        std::copy(dd, dd + 4, w.begin() + o);
        o += 4;
    }
    put(L.psl, psl);
    put(L.slong, h.sm_long);
    put(L.comb, h.comb);
    o = L.pdesc;  // pair item descriptors {g * n_pair + j, e0, e1, tp[lh][0]}
    for (int32_t it : h.pitems) {
        const int g = it / h.n_pair, j = it % h.n_pair, lh = lh_of_g(g);
        const int32_t* pp = &h.pp[(size_t)lh * (h.n_pair + 1)];
        const int32_t d[4] = {it, pp[j], pp[j + 1], h.tp[(size_t)lh * (h.n_rb + 1)]};
        std::copy(d, d + 4, w.begin() + o);
        o += 4;
    }
    if (h.pent.empty()) { w[L.pent] = 0; w[L.pent + 1] = -1; w[L.pent + 2] = -1; }
    put(L.pent, h.pent);
    put(L.pcta, h.pcta_ptr);
    o = L.fp;  // pair assignment as row-block item descriptors, per CTA
    std::vector<int32_t> fpcta(1, 0);
    for (size_t c = 0; c + 1 < h.pcta_ptr.size(); ++c) {
        for (int i = h.pcta_ptr[c]; i < h.pcta_ptr[c + 1]; ++i) {
            const int it = h.pitems[i], g = it / h.n_pair, j = it % h.n_pair;
            const int32_t* tp = &h.tp[(size_t)lh_of_g(g) * (h.n_rb + 1)];
            for (int rb = 2 * j; rb < std::min(2 * j + 2, h.n_rb); ++rb) {
                const int32_t d[4] = {g * h.n_rb + rb, tp[rb], tp[rb + 1], tp[0]};
                std::copy(d, d + 4, w.begin() + o);
                o += 4;
            }
        }
        fpcta.push_back((int32_t)((o - L.fp) / 4));
    }
    put(L.fpcta, fpcta);
    o = L.cdesc;  // column item descriptors {g * n_cb + c, e0, e1, tp[lh][0]}
    for (int32_t it : h.citems) {
        const int g = it / h.n_cb, c = it % h.n_cb, lh = lh_of_g(g);
        const int32_t* cp = &h.cpp[(size_t)lh * (h.n_cb + 1)];
        const int32_t d[4] = {it, cp[c], cp[c + 1], h.tp[(size_t)lh * (h.n_rb + 1)]};
        std::copy(d, d + 4, w.begin() + o);
        o += 4;
    }
    if (h.cent.empty()) { w[L.cent] = 0; w[L.cent + 1] = -1; w[L.cent + 2] = -1; }
    put(L.cent, h.cent);
    put(L.ccta, h.ccta_ptr);
    DevSched& d = db->rel;
    d.n_rb = h.n_rb;
    d.n_lh = h.n_lh;
    d.lh_mode = h.lh_mode;
    d.slots_per_head = h.slots_per_head;
    d.max_rb_tiles = h.max_rb_tiles;
    d.mean_rb_tiles = (int)((h.tinfo.size() + (size_t)h.n_lh * h.n_rb - 1) / ((size_t)h.n_lh * h.n_rb));
    d.n_items = (int)(desc.size() / 4);
    d.n_comb = split ? (int)(h.comb.size() / 4) : 0;
    d.n_sm_long = (int)h.sm_long.size();
    {   // the IR kernel's team classes over iri (longest first): 8 warps for > 4 * KR tiles, then 4, 2,
        // 1 (each warp merges <= KR tiles in registers); KR = kIrWarpTiles unless its CTAs need more
        // than one wave on n_sm SMs, then kIrWarpTilesWide
        auto lh_of_g2 = [&](int g) { return h0.lh_mode == LH_ONE ? 0 : (h0.lh_mode == LH_BATCH ? g / h0.H : g % h0.H); };
        auto classes = [&](int kr, int (&nc)[4]) {
            for (int c = 0; c < 4; ++c) nc[c] = 0;
            for (int32_t it : h0.items) {
                const int g = it / h0.n_rb, rb = it % h0.n_rb;
                const int32_t* tp = &h0.tp[(size_t)lh_of_g2(g) * (h0.n_rb + 1)];
                const int n = tp[rb + 1] - tp[rb];
                nc[n > 4 * kr ? 0 : n > 2 * kr ? 1 : n > kr ? 2 : 3]++;
            }
            int64_t ctas = 0;
            for (int c = 0; c < 4; ++c) ctas += (nc[c] + (1 << c) - 1) >> c;
            return ctas;
        };
        d.ir_warp_tiles = kIrWarpTiles;
        if (classes(kIrWarpTiles, d.n_ir_class) > (int64_t)kIrCtasPerSm * n_sm) {
            d.ir_warp_tiles = kIrWarpTilesWide;
            classes(kIrWarpTilesWide, d.n_ir_class);
        }
    }
    // fp32 SIMT kernels: the fewest threads per row that still give >= 2 CTAs per SM (each thread
    // then owns the most columns), else 32
    d.simt_tpr = 32;
    for (int tpr = 4; tpr < 32; tpr *= 2)
        if ((int64_t)d.n_items * tpr >= 2 * (int64_t)n_sm) { d.simt_tpr = tpr; break; }
    d.n_cta = (int)cta_ptr.size() - 1;
    d.n_pair = h.n_pair;
    d.n_pcta = (int)h.pcta_ptr.size() - 1;
    d.n_cb = h.n_cb;
    d.n_ccta = (int)h.ccta_ptr.size() - 1;
    return db;
}

// The device schedule with its pointers inside a workspace's schedule region.
DevSched place(const DevBlob& db, void* region, bool has_kv)
{
    int32_t* b = (int32_t*)region;
    const BlobLayout& L = db.L;
    DevSched d = db.rel;
    d.tp = b + L.tp;
    d.tinfo = b + L.tinfo;
    d.kv_len = has_kv ? b + L.kv : nullptr;
    d.item_desc = (const int4*)(b + L.desc);
    d.items = b + L.items;
    d.cta_ptr = b + L.cta;
    d.ir_desc = (const int4*)(b + L.iri);
    d.psl = b + L.psl;
    d.sm_long = b + L.slong;
    d.comb = (const int4*)(b + L.comb);
    d.pair_desc = (const int4*)(b + L.pdesc);
    d.pent = (const int4*)(b + L.pent);
    d.pcta_ptr = b + L.pcta;
    d.fp_desc = (const int4*)(b + L.fp);
    d.fpcta_ptr = b + L.fpcta;
    d.col_desc = (const int4*)(b + L.cdesc);
    d.cent = (const int4*)(b + L.cent);
    d.ccta_ptr = b + L.ccta;
    return d;
}

// Greedy longest-processing-time assignment of the (already longest-first) items to n_cta
// persistent CTAs: each item goes to the CTA with the least work so far.  Cost of an item =
// 2 x its tiles + 1 (the Q load / O store of a row-block is about half a tile's traffic).  Items
// are regrouped per CTA in assignment order, so the first wave is the round-robin one (neighbouring
// CTAs run items of the same head at the same time and share its K/V tiles in L2).
void lpt_assign(std::vector<int32_t>& items, const std::vector<int64_t>& cost, int n_cta, std::vector<int32_t>& cta_ptr)
{
    const size_t n = items.size();
    n_cta = (int)std::max<size_t>(1, std::min<size_t>(n, (size_t)std::max(n_cta, 1)));
    // longest first (stable: ties keep head-major order), then each to the least loaded CTA
    std::vector<size_t> order(n);
    for (size_t i = 0; i < n; ++i) order[i] = i;
    std::stable_sort(order.begin(), order.end(), [&](size_t a, size_t b) { return cost[a] > cost[b]; });
    std::vector<int> owner(n);
    std::vector<int32_t> count(n_cta, 0);
    using E = std::pair<int64_t, int>;  // (load, cta)
    std::priority_queue<E, std::vector<E>, std::greater<E>> pq;
    for (int c = 0; c < n_cta; ++c) pq.push({0, c});
    for (size_t i : order) {
        E e = pq.top();
        pq.pop();
        owner[i] = e.second;
        ++count[e.second];
        e.first += cost[i];
        pq.push(e);
    }
    cta_ptr.assign(n_cta + 1, 0);
    for (int c = 0; c < n_cta; ++c) cta_ptr[c + 1] = cta_ptr[c] + count[c];
    std::vector<int32_t> fill(cta_ptr.begin(), cta_ptr.end() - 1), out(n);
    for (size_t i : order) out[fill[owner[i]]++] = items[i];
    items.swap(out);
}

// Fixed cost of an item (Q load, row statistics, O store, pipeline fill) in units of half a tile
// (3: measured on the one-launch kernel, C2 25.8 -> 24.7 us; 1 and 6-10 are slower or equal);
// SR_LPT_FIXED overrides for experiments.
int64_t lpt_item_cost()
{
    static const int64_t v = [] { const char* e = getenv("SR_LPT_FIXED"); return e ? (int64_t)atoi(e) : (int64_t)3; }();
    return v;
}

// Per-CTA item ranges for both schedules.  Cost of an item = 2 x its tiles + 1 (the Q load / O
// store of a row-block is about half a tile's traffic); of a pair = its two row-blocks' tiles + 1.
void lpt_assign(HostSched& h, int n_cta)
{
    auto lh_of_g = [&](int g) { return h.lh_mode == LH_ONE ? 0 : (h.lh_mode == LH_BATCH ? g / h.H : g % h.H); };
    std::vector<int64_t> cost(h.items.size());
    for (size_t i = 0; i < h.items.size(); ++i) {
        const int g = h.items[i] / h.n_rb, rb = h.items[i] % h.n_rb;
        const int32_t* tp = &h.tp[(size_t)lh_of_g(g) * (h.n_rb + 1)];
        cost[i] = 2 * (int64_t)(tp[rb + 1] - tp[rb]) + lpt_item_cost();
    }
    lpt_assign(h.items, cost, n_cta, h.cta_ptr);
    std::vector<int64_t> pcost(h.pitems.size());
    for (size_t i = 0; i < h.pitems.size(); ++i) {
        const int g = h.pitems[i] / h.n_pair, j = h.pitems[i] % h.n_pair;
        const int32_t* tp = &h.tp[(size_t)lh_of_g(g) * (h.n_rb + 1)];
        const int rb1 = std::min(2 * j + 2, h.n_rb);
        pcost[i] = 2 * (int64_t)(tp[rb1] - tp[2 * j]) + 2 * lpt_item_cost();
    }
    lpt_assign(h.pitems, pcost, n_cta, h.pcta_ptr);
    std::vector<int64_t> ccost(h.citems.size());
    for (size_t i = 0; i < h.citems.size(); ++i) {
        const int g = h.citems[i] / h.n_cb, c = h.citems[i] % h.n_cb;
        const int32_t* cp = &h.cpp[(size_t)lh_of_g(g) * (h.n_cb + 1)];
        ccost[i] = 2 * (int64_t)(cp[c + 1] - cp[c]) + 1;
    }
    lpt_assign(h.citems, ccost, n_cta, h.ccta_ptr);
}

// The cached host schedule of a request (built on a miss; LRU-bounded, host memory only).
sr_status host_sched(const Request& r, std::shared_ptr<CachedSched>& out)
{
    std::string key = sched_key(r);
    {
        std::lock_guard<std::mutex> lk(g_mu);
        auto itc = g_cache.find(key);
        if (itc != g_cache.end()) {
            g_lru.splice(g_lru.begin(), g_lru, itc->second.second);
            out = itc->second.first;
            return SR_OK;
        }
    }
    auto cs = std::make_shared<CachedSched>();
    sr_status s = build_sched(r, cs->hs);
    if (s != SR_OK) return s;
    std::lock_guard<std::mutex> lk(g_mu);
    auto itc = g_cache.find(key);  // another thread may have inserted it meanwhile
    if (itc != g_cache.end()) {
        out = itc->second.first;
        return SR_OK;
    }
    g_lru.push_front(key);
    g_cache.emplace(key, std::make_pair(cs, g_lru.begin()));
    while (g_cache.size() > kCacheCap) {  // evict the least recently used (callers hold shared_ptrs)
        g_cache.erase(g_lru.back());
        g_lru.pop_back();
    }
    out = cs;
    return SR_OK;
}

// SM count of the current device (cached per device; no synchronisation).
sr_status device_sms(int& n_sm)
{
    static std::mutex mu;
    static std::map<int, int> sms;
    int dev = -1;
    cudaError_t ce = cudaGetDevice(&dev);
    if (ce != cudaSuccess) return fail(SR_ERR_CUDA, "cudaGetDevice: %s", cudaGetErrorString(ce));
    std::lock_guard<std::mutex> lk(mu);
    auto it = sms.find(dev);
    if (it == sms.end()) {
        int n = 0;
        if ((ce = cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess)
            return fail(SR_ERR_CUDA, "cudaDeviceGetAttribute: %s", cudaGetErrorString(ce));
        it = sms.emplace(dev, n).first;
    }
    n_sm = it->second;
    return SR_OK;
}

// L2 size of the current device in bytes (cached; 0 if unknown).
size_t device_l2_bytes()
{
    static std::mutex mu;
    static std::map<int, size_t> l2;
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess) return 0;
    std::lock_guard<std::mutex> lk(mu);
    auto it = l2.find(dev);
    if (it == l2.end()) {
        int n = 0;
        if (cudaDeviceGetAttribute(&n, cudaDevAttrL2CacheSize, dev) != cudaSuccess) n = 0;
        it = l2.emplace(dev, (size_t)n).first;
    }
    return it->second;
}

std::shared_ptr<DevBlob> device_blob(CachedSched& cs, int n_sm, bool split = false)
{
    std::lock_guard<std::mutex> lk(cs.mu);
    for (auto& b : cs.blobs)
        if (b->n_sm == n_sm && b->split == split) return b;
    cs.blobs.push_back(make_blob(cs.hs, n_sm, split));
    return cs.blobs.back();
}

double l2_or_default()
{
    const size_t l2 = device_l2_bytes();
    return l2 ? (double)l2 : 126.0 * (1 << 20);
}

// Enqueue the upload of the given blob groups into the workspace's schedule region (k_sched.cu).
cudaError_t upload(const DevBlob& db, void* region, unsigned groups, cudaStream_t st, int64_t* nl)
{
    size_t off[G_N], len[G_N];
    int n = 0;
    for (int g = 0; g < G_N; ++g)
        if (((groups >> g) & 1) && db.L.g_len[g]) {
            if (n && off[n - 1] + len[n - 1] == db.L.g_off[g]) {  // adjacent groups: one segment
                len[n - 1] += db.L.g_len[g];
                continue;
            }
            off[n] = db.L.g_off[g];
            len[n] = db.L.g_len[g];
            ++n;
        }
    return launch_sched_upload(region, db.w.data(), off, len, n, st, nl);
}

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

void ws_layout(const HostSched& h, int B, int H, int D, int in_dtype, int fused, sr_ws_info* info)
{
    memset(info, 0, sizeof(*info));
    info->tile_n = h.T;
    info->slots_per_head = h.slots_per_head;
    info->n_slots = (int64_t)B * H * h.slots_per_head;
    int elt = (in_dtype == SR_F32) ? 4 : 2;
    info->xprime_elt_bytes = elt;
    size_t tile_bytes = (size_t)kRowBlock * h.T * elt;
    size_t stat_bytes = (size_t)info->n_slots * kRowBlock * sizeof(float);
    size_t o = 0;
    // first: the call's tile schedule, uploaded into the workspace by every call (k_sched.cu); its
    // size depends only on the mask, so every mode of one request (recomposed, training) shares it
    info->sched_bytes = sched_region_bytes(h);
    info->off_sched = o; o = align_up(o + info->sched_bytes, 1024);
    info->off_xprime = o;
    o = align_up(o + (size_t)info->n_slots * tile_bytes, 1024);
    // fused: 1 recomposed (X' + statistics), 0 unfused (S + P), 2 SD (X' + S/Y + statistics),
    // 3 training (the recomposed layout, then dS' tiles and the backward's row statistics)
    if (fused == 0 || fused == 2) {
        info->off_p = o; o = align_up(o + (size_t)info->n_slots * tile_bytes, 1024);
    }
    if (fused) {
        info->off_mprime = o; o = align_up(o + stat_bytes, 1024);
        info->off_dprime = o; o = align_up(o + stat_bytes, 1024);
        info->off_rprime = o; o = align_up(o + stat_bytes, 1024);
        info->off_rowstat = o; o = align_up(o + (size_t)4 * B * H * h.n_rb * kRowBlock * sizeof(float), 1024);
    }
    if ((fused == 1 || fused == 3) && h.n_partial > 0) {  // SR_SPLIT_KV: fp32 partial outputs of split rows
        info->off_partial = o; o = align_up(o + (size_t)h.n_partial * kRowBlock * D * sizeof(float), 1024);
    }
    if (fused == 3) {
        info->off_ds = o; o = align_up(o + (size_t)info->n_slots * tile_bytes, 1024);
        info->off_bstat = o; o = align_up(o + (size_t)3 * B * H * h.n_rb * kRowBlock * sizeof(float), 1024);
    }
    info->total_bytes = o;
}

bool overlaps(const void* a, size_t na, const void* b, size_t nb)
{
    uintptr_t x = (uintptr_t)a, y = (uintptr_t)b;
    return x < y + nb && y < x + na;
}

sr_status run(sr_entry e, int fused, const void* q, const void* k, const void* v, void* out, int B,
              int H, int S, int D, float scale, const void* mask_or_layout, int causal,
              const sr_exec* ex)
{
    if (!ex) return fail(SR_ERR_INVALID, "exec descriptor is NULL");
    if (!q || !k || !v || !out) return fail(SR_ERR_INVALID, "q, k, v and out must be non-NULL");
    if (!std::isfinite(scale) || !(scale > 0.f)) return fail(SR_ERR_INVALID, "scale must be finite and > 0");
    const int variant_bits =
        SR_FUSE_IR | SR_DECOMPOSE | SR_IR_KERNEL | SR_ONE_KERNEL | SR_TWO_KERNELS | SR_SPLIT_KV | SR_CONCURRENT;
    if (ex->flags & ~(SR_RUN_GEMM1 | SR_RUN_REDUCE | SR_RUN_GEMM2 | SR_GS_PROLOGUE | SR_SCHED_RESIDENT | variant_bits))
        return fail(SR_ERR_INVALID, "unknown flags 0x%x", ex->flags);
    if ((ex->flags & variant_bits) && (!fused || ex->in_dtype == SR_F32))
        return fail(SR_ERR_UNSUPPORTED, "SR_FUSE_IR / SR_DECOMPOSE / SR_IR_KERNEL apply to the recomposed 16-bit path only");
    {
        const int v = ex->flags & variant_bits;
        if (v & (v - 1)) return fail(SR_ERR_INVALID, "SR_FUSE_IR, SR_DECOMPOSE, SR_IR_KERNEL and SR_ONE_KERNEL are exclusive");
    }
    // the one-launch kernel: asked for, or the 16-bit recomposed default at T = 64 (any tile_n = 128
    // request without a variant bit runs the two-kernel chain at T = 128)
    bool one = (ex->flags & SR_ONE_KERNEL) != 0;
    if (one && ex->tile_n != 0 && ex->tile_n != 64) return fail(SR_ERR_UNSUPPORTED, "SR_ONE_KERNEL uses T = 64");
    const bool conc_req = (ex->flags & SR_CONCURRENT) != 0;
    if (conc_req && ((ex->tile_n != 0 && ex->tile_n != 64) ||
                     (ex->flags & (SR_RUN_GEMM1 | SR_RUN_REDUCE | SR_RUN_GEMM2))))
        return fail(SR_ERR_UNSUPPORTED, "SR_CONCURRENT runs T = 64, whole layers only");
    if (conc_req) one = true;  // same workspace and schedule as the one-launch default
    if (fused == 1 && ex->in_dtype != SR_F32 && !(ex->flags & variant_bits) && (ex->tile_n == 0 || ex->tile_n == 64))
        one = true;
    if (fused && (ex->flags & SR_DECOMPOSE)) fused = 2;  // SD: workspace mode 2
    Request r;
    sr_status s = check_request(e, B, H, S, D, ex->in_dtype, mask_or_layout, causal, one ? 64 : ex->tile_n, r, fused);
    if (s != SR_OK) return s;
    if (ex->out_dtype != ex->in_dtype && ex->out_dtype != SR_F32)
        return fail(SR_ERR_UNSUPPORTED, "out_dtype must equal in_dtype or be SR_F32");
    if (!fused && ex->in_dtype == SR_F32)
        return fail(SR_ERR_UNSUPPORTED, "the unfused baseline runs 16-bit dtypes only");
    size_t in_bytes = (size_t)B * H * S * D * dtype_bytes(ex->in_dtype);
    size_t out_bytes = (size_t)B * H * S * D * dtype_bytes(ex->out_dtype);
    if (overlaps(out, out_bytes, q, in_bytes) || overlaps(out, out_bytes, k, in_bytes) ||
        overlaps(out, out_bytes, v, in_bytes))
        return fail(SR_ERR_INVALID, "out overlaps q, k or v");
    if (((uintptr_t)q | (uintptr_t)k | (uintptr_t)v | (uintptr_t)out) & 15)
        return fail(SR_ERR_INVALID, "q, k, v, out must be 16-byte aligned");
    std::shared_ptr<CachedSched> cs;
    s = host_sched(r, cs);  // host-only schedule: workspace checks precede any CUDA call
    if (s != SR_OK) return s;
    sr_ws_info wi;
    ws_layout(cs->hs, B, H, D, ex->in_dtype, fused, &wi);
    if (!ex->workspace || ex->workspace_bytes < wi.total_bytes)
        return fail(SR_ERR_WORKSPACE, "workspace %zu bytes < required %zu", ex->workspace_bytes, wi.total_bytes);
    if ((uintptr_t)ex->workspace & 255) return fail(SR_ERR_WORKSPACE, "workspace must be 256-byte aligned");
    int n_sm = 0;
    if ((s = device_sms(n_sm)) != SR_OK) return s;
    // key-range split: asked for, or chosen for the default 16-bit path when a few long rows would
    // dominate the one-launch schedule (most loaded CTA >= 3x a balanced share, rows of >= 32 tiles:
    // e.g. one GPU's share of a head-sharded BigBird / Longformer layer, whose global rows hold every
    // key tile; measured C4 / C5 at 8-way sharding 50.3 -> 38.5 / 52.4 -> 30.7 us, while causal C3
    // shards and all full configs stay faster in one launch).  SR_SPLIT_AUTO=0 disables the choice.
    bool split = (ex->flags & SR_SPLIT_KV) != 0;
    if (!split && fused == 1 && one && !(ex->flags & (variant_bits | SR_RUN_GEMM1 | SR_RUN_REDUCE | SR_RUN_GEMM2)) &&
        cs->hs.n_partial > 0 && cs->hs.max_rb_tiles >= 32) {
        static const bool auto_split = [] { const char* e = getenv("SR_SPLIT_AUTO"); return !e || atoi(e) != 0; }();
        if (auto_split && device_blob(*cs, n_sm, false)->imbalance >= 3.0) {
            split = true;
            one = false;
        }
    }
    // the concurrent GEMM1 / GEMM2 kernel (k_conc.cu) runs only when asked for (SR_CONCURRENT):
    // measured slower than the one-launch default on every config
    const bool conc = conc_req;
    std::shared_ptr<DevBlob> db = device_blob(*cs, n_sm, split);
    void* region = (char*)ex->workspace + wi.off_sched;

    Params p{};
    p.q = q; p.k = k; p.v = v; p.out = out;
    p.B = B; p.H = H; p.S = S; p.Spad = (S + kRowBlock - 1) / kRowBlock * kRowBlock; p.D = D; p.T = r.T;
    p.scale = scale;
    p.scale_log2 = scale * 1.4426950408889634f;
    p.causal = r.causal;
    p.mask_kind = e == SR_E_WINDOW ? MK_WINDOW : (e == SR_E_BLOCKSPARSE ? MK_BLOCK : MK_DENSE);
    p.win_half = r.window / 2;
    p.n_global = r.n_global;
    p.in_dtype = ex->in_dtype;
    p.out_dtype = ex->out_dtype;
    p.sc = place(*db, region, r.kv_len != nullptr);
    const int stage_bits = ex->flags & (SR_RUN_GEMM1 | SR_RUN_REDUCE | SR_RUN_GEMM2);
    p.stages = stage_bits ? stage_bits : (SR_RUN_GEMM1 | SR_RUN_REDUCE | SR_RUN_GEMM2);
    p.ir_mode = (ex->flags & SR_FUSE_IR) ? IR_IN_GEMM2 : (((ex->flags & SR_IR_KERNEL) || split) ? IR_KERNEL : IR_IN_GEMM1);
    {   // GEMM1 pair schedule: SR_G1_PAIR=0/1 overrides the default (experiments)
        static const int env_pair = [] { const char* e = getenv("SR_G1_PAIR"); return e ? atoi(e) : -1; }();
        // default: pairs when K tiles are as large as the X' tiles they produce (D = 128), there are
        // enough pairs to keep every SM busy, and the two row-blocks of a pair share most of their K
        // tiles (>= 45 % of the K loads saved: causal dense layers from S ~ 1536 on; measured one
        // B200, back to back: causal S = 4096 572 -> 531 us, C3 136.0 -> 134.4; banded layouts lose --
        // GPT-Neo local S = 2048 window 510 58.1 -> 66.2 us, window 254 47.0 -> 73.2 -- and stay unpaired;
        // D = 64 configs lose)
        p.g1_pair = env_pair >= 0 ? env_pair : (D == 128 && p.sc.n_pcta > 0 &&
                                                 (int64_t)B * H * p.sc.n_pair >= 2 * (int64_t)p.sc.n_pcta &&
                                                 cs->hs.pair_saving >= 0.45);
        if (split || conc) p.g1_pair = 0;  // chunks of row-blocks, not pairs / row-block items

    }
    {   // X' (or S) stores stream past L2 (evict_first) only when the layer's stored tiles exceed
        // half the device's L2; below that they keep normal priority and are read back from L2
        // (measured, one B200, back-to-back: C2 (31.5 MB of X') 18.5 -> 17.6 us; C5 (132 MB) slower
        // without the hint).  SR_X_EVICT_FIRST=0/1 overrides (experiments).
        static const int env_x = [] { const char* e = getenv("SR_X_EVICT_FIRST"); return e ? atoi(e) : -1; }();
        const double x_bytes = (double)cs->hs.stored_elems * (ex->in_dtype == SR_F32 ? 4.0 : 2.0);
        p.x_evict_first = env_x >= 0 ? env_x : (x_bytes > 0.5 * l2_or_default());
        if (conc && env_x < 0) p.x_evict_first = 0;  // GEMM2 reads each item's X' back soon after it is written
    }
    char* ws = (char*)ex->workspace;
    p.xprime = ws + wi.off_xprime;
    if (fused) {
        p.mprime = (float*)(ws + wi.off_mprime);
        p.dprime = (float*)(ws + wi.off_dprime);
        p.rprime = (float*)(ws + wi.off_rprime);
        p.rowstat = (float*)(ws + wi.off_rowstat);
    }
    if (fused != 1) p.pbuf = ws + wi.off_p;
    p.partial = split ? (float*)(ws + wi.off_partial) : nullptr;
    cudaStream_t st = (cudaStream_t)ex->stream;
    int64_t nl = 0;
    cudaError_t ce;
    // the schedule groups this call's kernels read, uploaded into the workspace ahead of them
    const bool one_pair = fused == 1 && one && p.g1_pair;
    const unsigned groups = one_pair ? (1u << G_BASE | 1u << G_PAIR | 1u << G_FP)
                                     : (1u << G_BASE | 1u << G_ITEMS | (p.g1_pair ? 1u << G_PAIR : 0u) |
                                        (!fused && !cs->hs.sm_long.empty() ? 1u << G_SML : 0u));
    if (!(ex->flags & SR_SCHED_RESIDENT) && (ce = upload(*db, region, groups, st, &nl)) != cudaSuccess) {
        g_launches += nl;
        return fail(SR_ERR_CUDA, "schedule upload: %s", cudaGetErrorString(ce));
    }
    if (fused == 2) {
        ce = launch_tc_sd(p, st, &nl);
    } else if (conc) {
        ce = launch_tc_conc(p, st, &nl);
    } else if (fused && one) {
        // pairs of row-blocks sharing each K tile in phase 1 (same choice as the two-kernel chain:
        // D = 128 with enough pairs); phase 2 then walks the pair assignment as row-block items
        if (p.g1_pair) {
            p.sc.item_desc = p.sc.fp_desc;
            p.sc.cta_ptr = p.sc.fpcta_ptr;
            p.sc.n_cta = p.sc.n_pcta;
        }
        p.gs_prologue = (ex->flags & SR_GS_PROLOGUE) != 0;
        {   // read part of X' back from L2: phase 2 walks the CTA's items last-first (the X' phase 1
            // wrote most recently is the likeliest still in L2) and the last 2 items' X' is stored
            // without the evict_first hint (measured, one B200, burst / sustained under the power cap:
            // C3 140.5 -> 136.7 / 164.0 -> 158.7 us, C4 120.1 -> 115.3 / 141.2 -> 138.9, C5 63.6 -> 60.0 /
            // 70.8 -> 68.5).  SR_X_KEEP / SR_P2_REVERSE override (experiments).
            static const int env_keep = [] { const char* e = getenv("SR_X_KEEP"); return e ? atoi(e) : 2; }();
            static const int env_rev = [] { const char* e = getenv("SR_P2_REVERSE"); return e ? atoi(e) : 1; }();
            static const int env_rev1 = [] { const char* e = getenv("SR_P1_REVERSE"); return e ? atoi(e) : 0; }();
            p.x_keep = env_keep;
            p.p2_reverse = env_rev1 ? 0 : env_rev;
            p.p1_reverse = env_rev1;
        }

        ce = launch_tc_one(p, st, &nl);
    } else if (fused) {
        ce = ex->in_dtype == SR_F32 ? launch_simt_f32(p, st, &nl) : launch_tc_fused(p, st, &nl);
    } else {
        ce = launch_tc_unfused(p, st, &nl);
    }
    g_launches += nl;
    if (ce != cudaSuccess) return fail(SR_ERR_CUDA, "kernel launch: %s", cudaGetErrorString(ce));
    return SR_OK;
}

// Training backward (include/sr_mha.h): validation, then prep -> dS' -> dQ ->
// dK -> dV on the forward's workspace.
sr_status run_bwd(sr_entry e, const void* q, const void* k, const void* v, const void* out, const void* dout,
                  void* dq, void* dk, void* dv, int B, int H, int S, int D, float scale, const void* mask_or_layout,
                  int causal, const sr_exec* ex)
{
    if (!ex) return fail(SR_ERR_INVALID, "exec descriptor is NULL");
    if (!q || !k || !v || !out || !dout || !dq || !dk || !dv)
        return fail(SR_ERR_INVALID, "q, k, v, out, dout, dq, dk and dv must be non-NULL");
    if (!std::isfinite(scale) || !(scale > 0.f)) return fail(SR_ERR_INVALID, "scale must be finite and > 0");
    if (ex->flags & ~(SR_RUN_GEMM1 | SR_RUN_REDUCE | SR_RUN_GEMM2 | SR_SCHED_RESIDENT))
        return fail(SR_ERR_INVALID, "backward flags must be SR_RUN_* stage bits or SR_SCHED_RESIDENT (got 0x%x)",
                    ex->flags);
    Request r;
    sr_status s = check_request(e, B, H, S, D, ex->in_dtype, mask_or_layout, causal, ex->tile_n, r, 3);
    if (s != SR_OK) return s;
    if (ex->in_dtype == SR_F32) return fail(SR_ERR_UNSUPPORTED, "the backward runs 16-bit dtypes only");
    if (ex->out_dtype != ex->in_dtype && ex->out_dtype != SR_F32)
        return fail(SR_ERR_UNSUPPORTED, "out_dtype must equal in_dtype or be SR_F32");
    const size_t in_bytes = (size_t)B * H * S * D * dtype_bytes(ex->in_dtype);
    const size_t out_bytes = (size_t)B * H * S * D * dtype_bytes(ex->out_dtype);
    const void* ins[5] = {q, k, v, dout, out};
    const size_t ins_b[5] = {in_bytes, in_bytes, in_bytes, in_bytes, out_bytes};
    void* gs[3] = {dq, dk, dv};
    for (int a = 0; a < 3; ++a) {
        for (int b = 0; b < 5; ++b)
            if (overlaps(gs[a], out_bytes, ins[b], ins_b[b])) return fail(SR_ERR_INVALID, "a gradient overlaps an input");
        for (int b = a + 1; b < 3; ++b)
            if (overlaps(gs[a], out_bytes, gs[b], out_bytes)) return fail(SR_ERR_INVALID, "gradients overlap");
    }
    if (((uintptr_t)q | (uintptr_t)k | (uintptr_t)v | (uintptr_t)out | (uintptr_t)dout | (uintptr_t)dq |
         (uintptr_t)dk | (uintptr_t)dv) & 15)
        return fail(SR_ERR_INVALID, "all tensors must be 16-byte aligned");
    std::shared_ptr<CachedSched> cs;
    s = host_sched(r, cs);
    if (s != SR_OK) return s;
    sr_ws_info wi;
    ws_layout(cs->hs, B, H, D, ex->in_dtype, 3, &wi);
    if (!ex->workspace || ex->workspace_bytes < wi.total_bytes)
        return fail(SR_ERR_WORKSPACE, "workspace %zu bytes < required %zu (SR_WS_TRAIN)", ex->workspace_bytes,
                    wi.total_bytes);
    if ((uintptr_t)ex->workspace & 255) return fail(SR_ERR_WORKSPACE, "workspace must be 256-byte aligned");
    int n_sm = 0;
    if ((s = device_sms(n_sm)) != SR_OK) return s;
    std::shared_ptr<DevBlob> db = device_blob(*cs, n_sm);
    void* region = (char*)ex->workspace + wi.off_sched;

    Params p{};
    p.q = q; p.k = k; p.v = v; p.out = const_cast<void*>(out);
    p.B = B; p.H = H; p.S = S; p.Spad = (S + kRowBlock - 1) / kRowBlock * kRowBlock; p.D = D; p.T = r.T;
    p.scale = scale;
    p.scale_log2 = scale * 1.4426950408889634f;
    p.causal = r.causal;
    p.mask_kind = e == SR_E_WINDOW ? MK_WINDOW : (e == SR_E_BLOCKSPARSE ? MK_BLOCK : MK_DENSE);
    p.win_half = r.window / 2;
    p.n_global = r.n_global;
    p.in_dtype = ex->in_dtype;
    p.out_dtype = ex->out_dtype;
    p.sc = place(*db, region, r.kv_len != nullptr);
    const int stage_bits = ex->flags & (SR_RUN_GEMM1 | SR_RUN_REDUCE | SR_RUN_GEMM2);
    p.stages = stage_bits ? stage_bits : (SR_RUN_GEMM1 | SR_RUN_REDUCE | SR_RUN_GEMM2);
    p.ir_mode = IR_IN_GEMM1;
    char* ws = (char*)ex->workspace;
    p.xprime = ws + wi.off_xprime;
    p.mprime = (float*)(ws + wi.off_mprime);
    p.dprime = (float*)(ws + wi.off_dprime);
    p.rprime = (float*)(ws + wi.off_rprime);
    p.rowstat = (float*)(ws + wi.off_rowstat);
    p.dout = dout;
    p.dq = dq; p.dk = dk; p.dv = dv;
    p.dsbuf = ws + wi.off_ds;
    {   // X' reads and dS' stores stream past L2 only when the layer's stored X' + dS' tiles exceed
        // ~4/5 of the device's L2 (measured: C2, 63 MB, backward 50.1 -> 48.2-49.5 us at normal
        // priority; C5 unchanged)
        static const int env_x = [] { const char* e = getenv("SR_X_EVICT_FIRST"); return e ? atoi(e) : -1; }();
        const double xds_bytes = 2.0 * (double)cs->hs.stored_elems * 2.0;
        p.x_evict_first = env_x >= 0 ? env_x : (xds_bytes > 0.8 * l2_or_default());
    }
    p.bstat = (float*)(ws + wi.off_bstat);
    {   // dQ inside the dS' kernel (default); SR_BWD_DQ_SEPARATE=1 keeps the separate GEMM2-based dQ kernel
        static const bool sep = [] { const char* e = getenv("SR_BWD_DQ_SEPARATE"); return e && atoi(e) != 0; }();
        p.bwd_dq_fused = sep ? 0 : 1;
    }
    int64_t nl = 0;
    cudaError_t ce = cudaSuccess;
    if (!(ex->flags & SR_SCHED_RESIDENT))
        ce = upload(*db, region, 1u << G_BASE | 1u << G_ITEMS | 1u << G_COL, (cudaStream_t)ex->stream, &nl);
    if (ce == cudaSuccess) ce = launch_tc_bwd(p, (cudaStream_t)ex->stream, &nl);
    g_launches += nl;
    if (ce != cudaSuccess) return fail(SR_ERR_CUDA, "kernel launch: %s", cudaGetErrorString(ce));
    return SR_OK;
}

}  // namespace

// ================================================================================== C ABI

// One NVTX range per layer call: the host-side span of the call, named after the entry
// point; free when no profiler is attached.
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

extern "C" {

sr_status sr_mha_dense(const void* q, const void* k, const void* v, void* out, int B, int H, int S,
                       int D, float scale, const sr_dense_mask* m, int causal, const sr_exec* ex)
{
    NvtxRange nvtx("sr_mha_dense");
    return run(SR_E_DENSE, 1, q, k, v, out, B, H, S, D, scale, m, causal, ex);
}
sr_status sr_mha_blocksparse(const void* q, const void* k, const void* v, void* out, int B, int H,
                             int S, int D, float scale, const sr_block_layout* l, int causal,
                             const sr_exec* ex)
{
    NvtxRange nvtx("sr_mha_blocksparse");
    return run(SR_E_BLOCKSPARSE, 1, q, k, v, out, B, H, S, D, scale, l, causal, ex);
}
sr_status sr_mha_sliding_window(const void* q, const void* k, const void* v, void* out, int B,
                                int H, int S, int D, float scale, const sr_window* w, int causal,
                                const sr_exec* ex)
{
    NvtxRange nvtx("sr_mha_sliding_window");
    return run(SR_E_WINDOW, 1, q, k, v, out, B, H, S, D, scale, w, causal, ex);
}
sr_status sr_mha_dense_unfused(const void* q, const void* k, const void* v, void* out, int B,
                               int H, int S, int D, float scale, const sr_dense_mask* m, int causal,
                               const sr_exec* ex)
{
    NvtxRange nvtx("sr_mha_dense_unfused");
    return run(SR_E_DENSE, 0, q, k, v, out, B, H, S, D, scale, m, causal, ex);
}
sr_status sr_mha_blocksparse_unfused(const void* q, const void* k, const void* v, void* out, int B,
                                     int H, int S, int D, float scale, const sr_block_layout* l,
                                     int causal, const sr_exec* ex)
{
    NvtxRange nvtx("sr_mha_blocksparse_unfused");
    return run(SR_E_BLOCKSPARSE, 0, q, k, v, out, B, H, S, D, scale, l, causal, ex);
}
sr_status sr_mha_sliding_window_unfused(const void* q, const void* k, const void* v, void* out,
                                        int B, int H, int S, int D, float scale, const sr_window* w,
                                        int causal, const sr_exec* ex)
{
    NvtxRange nvtx("sr_mha_sliding_window_unfused");
    return run(SR_E_WINDOW, 0, q, k, v, out, B, H, S, D, scale, w, causal, ex);
}

sr_status sr_mha_dense_bwd(const void* q, const void* k, const void* v, const void* out, const void* dout,
                           void* dq, void* dk, void* dv, int B, int H, int S, int D, float scale,
                           const sr_dense_mask* m, int causal, const sr_exec* ex)
{
    NvtxRange nvtx("sr_mha_dense_bwd");
    return run_bwd(SR_E_DENSE, q, k, v, out, dout, dq, dk, dv, B, H, S, D, scale, m, causal, ex);
}
sr_status sr_mha_blocksparse_bwd(const void* q, const void* k, const void* v, const void* out, const void* dout,
                                 void* dq, void* dk, void* dv, int B, int H, int S, int D, float scale,
                                 const sr_block_layout* l, int causal, const sr_exec* ex)
{
    NvtxRange nvtx("sr_mha_blocksparse_bwd");
    return run_bwd(SR_E_BLOCKSPARSE, q, k, v, out, dout, dq, dk, dv, B, H, S, D, scale, l, causal, ex);
}
sr_status sr_mha_sliding_window_bwd(const void* q, const void* k, const void* v, const void* out, const void* dout,
                                    void* dq, void* dk, void* dv, int B, int H, int S, int D, float scale,
                                    const sr_window* w, int causal, const sr_exec* ex)
{
    NvtxRange nvtx("sr_mha_sliding_window_bwd");
    return run_bwd(SR_E_WINDOW, q, k, v, out, dout, dq, dk, dv, B, H, S, D, scale, w, causal, ex);
}

sr_status sr_workspace_query(sr_entry e, int fused, int B, int H, int S, int D, sr_dtype in_dtype,
                             const void* mask_or_layout, int causal, int tile_n, sr_ws_info* info)
{
    if (!info) return fail(SR_ERR_INVALID, "info is NULL");
    if (fused < 0 || fused > 3) return fail(SR_ERR_INVALID, "workspace mode %d must be 0..3", fused);
    if (fused == 3 && in_dtype == SR_F32) return fail(SR_ERR_UNSUPPORTED, "the backward runs 16-bit dtypes only");
    Request r;
    sr_status s = check_request(e, B, H, S, D, in_dtype, mask_or_layout, causal, tile_n, r, fused);
    if (s != SR_OK) return s;
    std::shared_ptr<CachedSched> cs;
    s = host_sched(r, cs);
    if (s != SR_OK) return s;
    ws_layout(cs->hs, B, H, D, in_dtype, fused, info);
    return SR_OK;
}

size_t sr_workspace_bytes(sr_entry e, int fused, int B, int H, int S, int D, sr_dtype in_dtype,
                          const void* mask_or_layout, int causal, int tile_n)
{
    sr_ws_info info;
    if (sr_workspace_query(e, fused, B, H, S, D, in_dtype, mask_or_layout, causal, tile_n, &info) != SR_OK)
        return 0;
    return info.total_bytes;
}

sr_status sr_schedule_stats(sr_entry e, int B, int H, int S, const void* mask_or_layout, int causal,
                            int tile_n, int64_t* n_tiles, int64_t* stored_elems)
{
    Request r;
    sr_status s = check_request(e, B, H, S, 64, SR_F16, mask_or_layout, causal, tile_n, r, 1);
    if (s != SR_OK) return s;
    std::shared_ptr<CachedSched> cs;
    s = host_sched(r, cs);
    if (s != SR_OK) return s;
    if (n_tiles) *n_tiles = cs->hs.n_tiles;
    if (stored_elems) *stored_elems = cs->hs.stored_elems;
    return SR_OK;
}

const char* sr_status_string(sr_status s)
{
    switch (s) {
    case SR_OK: return "SR_OK";
    case SR_ERR_INVALID: return "SR_ERR_INVALID";
    case SR_ERR_UNSUPPORTED: return "SR_ERR_UNSUPPORTED";
    case SR_ERR_WORKSPACE: return "SR_ERR_WORKSPACE";
    case SR_ERR_CUDA: return "SR_ERR_CUDA";
    }
    return "SR_?";
}

const char* sr_last_error(void) { return g_err; }
int64_t sr_launch_count(void) { return g_launches.load(); }
const char* sr_version(void) { return "sr_mha 0.1 (sm_100a)"; }

}  // extern "C"
