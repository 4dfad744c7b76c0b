// k_softmax.cu -- the unfused baseline's softmax kernel (a row vector per thread
// block held in on-chip memory; reads the attention matrix once and writes it once).  Part of the
// in-repo traffic baseline only; the recomposed path never runs it.
#include "tc_common.cuh"

namespace sr {

using namespace ptx;

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
}

template <int T>
cudaError_t launch_softmax_t(const Params& p, cudaStream_t st, int64_t* nl)
{
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    const size_t sm = 4 * (size_t)p.S * 2;
    cudaError_t e = cudaFuncSetAttribute(row_softmax<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    row_softmax<T><<<(unsigned)((rows + 3) / 4), 128, sm, st>>>(p);
    ++*nl;
    return cudaGetLastError();
}

cudaError_t launch_softmax(const Params& p, cudaStream_t st, int64_t* nl)
{
    return p.T == 64 ? launch_softmax_t<64>(p, st, nl) : launch_softmax_t<128>(p, st, nl);
}

}  // namespace sr
