// k_sd.cu -- SD: the softmax decomposition WITHOUT fusion (evaluated as "SD" in
// Fig. 8 / L219): GEMM1 writes the scaled, masked scores S; a standalone LS kernel reads S and
// writes X' = e^{x - m'} with m', d'; the IR kernel merges the statistics; a standalone GS kernel
// reads X' and r' and writes Y = X' r'; GEMM2 reads Y.  Six attention-matrix passes instead of the
// unfused baseline's four and SDF's two -- the paper's ladder baseline -> SD -> SDF.
//
// Both kernels are memory-bound row sweeps: one warp per (tile, row); a row of a tile is one
// 128-byte piece per 64 keys of the SWIZZLE_128B tile layout (lane l holds 2 values per piece;
// max and sum are warp-shuffle reductions; order inside the row does not matter).
#include "tc_common.cuh"

namespace sr {

using namespace ptx;

// (slot, row) -> is the row's 64-row half valid in that tile?  Slots past the end of a head's list
// (lists of different lengths per layout head) are unused.
__device__ __forceinline__ bool slot_row_valid(const Params& p, int64_t slot, int r)
{
    const DevSched& sc = p.sc;
    const int g = (int)(slot / sc.slots_per_head);
    const int local = (int)(slot % sc.slots_per_head);
    const int lh = lh_of(sc, g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    const int t = __ldg(tp) + local;
    if (t >= __ldg(tp + sc.n_rb)) return false;
    return (tinfo_half(__ldg(sc.tinfo + t)) >> (r / kHalf)) & 1;
}

template <int T>
__global__ void __launch_bounds__(256) sd_ls_kernel(const Params p, int64_t n_rows)
{
    ptx::griddep_launch_dependents();
    ptx::griddep_wait();
    const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32;
    const int lane = threadIdx.x % 32;
    if (wid >= n_rows) return;
    const int64_t slot = wid / kRowBlock;
    const int r = (int)(wid % kRowBlock);
    if (!slot_row_valid(p, slot, r)) return;
    constexpr int XB = kRowBlock * T * 2, NP = T / 64;
    const uint8_t* S = (const uint8_t*)p.pbuf + slot * (int64_t)XB;  // scores S (from GEMM1, plain)
    uint8_t* X = (uint8_t*)p.xprime + slot * (int64_t)XB;
    uint32_t w[NP];
    float mx = -INFINITY;
#pragma unroll
    for (int c = 0; c < NP; ++c) {
        w[c] = *reinterpret_cast<const uint32_t*>(S + c * (kRowBlock * 128) + r * 128 + lane * 4);
        const float2 f = unpack_f16(w[c]);
        mx = fmaxf(mx, fmaxf(f.x, f.y));
    }
    for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    const float l2e = 1.4426950408889634f, neg = (mx == -INFINITY) ? 0.f : -mx * l2e;
    float sum = 0.f;
#pragma unroll
    for (int c = 0; c < NP; ++c) {  // LS: X' = e^{x - m'}
        const float2 f = unpack_f16(w[c]);
        const float y0 = ex2(fmaf(f.x, l2e, neg)), y1 = ex2(fmaf(f.y, l2e, neg));
        sum += y0 + y1;
        *reinterpret_cast<uint32_t*>(X + c * (kRowBlock * 128) + r * 128 + lane * 4) = pack_f16(y0, y1);
    }
    for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
    if (lane == 0) {
        p.mprime[slot * kRowBlock + r] = mx;  // scores already carry the scale: natural-log units
        p.dprime[slot * kRowBlock + r] = sum;
    }
}

template <int T>
__global__ void __launch_bounds__(256) sd_gs_kernel(const Params p, int64_t n_rows)
{
    ptx::griddep_launch_dependents();
    ptx::griddep_wait();
    const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32;
    const int lane = threadIdx.x % 32;
    if (wid >= n_rows) return;
    const int64_t slot = wid / kRowBlock;
    const int r = (int)(wid % kRowBlock);
    if (!slot_row_valid(p, slot, r)) return;
    constexpr int XB = kRowBlock * T * 2, NP = T / 64;
    const uint8_t* X = (const uint8_t*)p.xprime + slot * (int64_t)XB;
    // Y = X' * r' goes into the S region (no longer needed after LS); GEMM2 reads it from there
    uint8_t* Y = (uint8_t*)p.pbuf + slot * (int64_t)XB;
    const float rr = __ldg(p.rprime + slot * kRowBlock + r);
    const bool bf = p.in_dtype == DT_BF16;
#pragma unroll
    for (int c = 0; c < NP; ++c) {  // GS: element-wise scaling by the row's reconstruction factor
        const size_t off = c * (kRowBlock * 128) + r * 128 + lane * 4;
        const float2 f = unpack_f16(*reinterpret_cast<const uint32_t*>(X + off));
        *reinterpret_cast<uint32_t*>(Y + off) = bf ? pack_bf16(f.x * rr, f.y * rr) : pack_f16(f.x * rr, f.y * rr);
    }
}

cudaError_t launch_gemm1(const Params& p, bool ls, cudaStream_t st, int64_t* nl);
cudaError_t launch_gemm2(const Params& p, int mode, cudaStream_t st, int64_t* nl);

template <int T>
cudaError_t launch_sd_t(const Params& p, cudaStream_t st, int64_t* nl)
{
    const int64_t n_rows = (int64_t)p.B * p.H * p.sc.slots_per_head * kRowBlock;
    const unsigned blocks = (unsigned)((n_rows * 32 + 255) / 256);
    cudaError_t e = cudaSuccess;
    if (p.stages & 2) {
        if ((e = launch_pdl(sd_ls_kernel<T>, dim3(blocks), dim3(256), 0, st, nl, p, n_rows)) != cudaSuccess) return e;
        if ((e = launch_ir(p, st, nl)) != cudaSuccess) return e;
        if ((e = launch_pdl(sd_gs_kernel<T>, dim3(blocks), dim3(256), 0, st, nl, p, n_rows)) != cudaSuccess) return e;
    }
    if (p.stages & 4) e = launch_gemm2(p, 0, st, nl);  // plain GEMM2 on Y (in pbuf)
    return e;
}

// SD workspace: pbuf holds S (written by the plain GEMM1) and then Y (read by the plain GEMM2),
// xprime holds X', plus the statistics.  Stage bits: GEMM1 / LS+IR+GS / GEMM2.
cudaError_t launch_tc_sd(const Params& p, cudaStream_t st, int64_t* nl)
{
    cudaError_t e = cudaSuccess;
    if (p.stages & 1) {
        Params g1 = p;
        g1.xprime = p.pbuf;  // the plain GEMM1 writes its score tiles where xprime points
        if ((e = launch_gemm1(g1, false, st, nl)) != cudaSuccess) return e;
    }
    return p.T == 64 ? launch_sd_t<64>(p, st, nl) : launch_sd_t<128>(p, st, nl);
}

}  // namespace sr
