// k_sd.cu -- SD: the softmax decomposition WITHOUT fusion (evaluated as "SD" in
// Fig. 8 / L219): GEMM1 writes the scaled, masked scores S; a standalone LS kernel reads S and
// writes X' = e^{x - m'} with m', d'; the IR kernel merges the statistics; a standalone GS kernel
// reads X' and r' and writes Y = X' r'; GEMM2 reads Y.  Six attention-matrix passes instead of the
// unfused baseline's four and SDF's two -- the paper's ladder baseline -> SD -> SDF.
//
// Both kernels are memory-bound tile sweeps: one CTA (4 warps) per slot pulls the tile (16 or 32
// KB, contiguous) into shared memory with one bulk copy, each warp rewrites the 32 rows of its own
// 64-row half in place (a row's 64-key chunk is one 128-B line; lane l holds 2 keys of each; max
// and sum are warp-shuffle reductions), and the valid halves go back out with bulk stores.
#include "tc_common.cuh"

namespace sr {

using namespace ptx;

template <int T, bool LS>
__global__ void __launch_bounds__(128) sd_tile_kernel(const Params p)
{
    constexpr int XB = kRowBlock * T * 2, NP = T / 64;
    __shared__ __align__(128) uint8_t tile[XB];
    __shared__ uint64_t bar;
    const int64_t slot = blockIdx.x;
    const DevSched& sc = p.sc;
    const int g = (int)(slot / sc.slots_per_head);
    const int local = (int)(slot % sc.slots_per_head);
    const int32_t* tp = sc.tp + (size_t)lh_of(sc, g, p.H) * (sc.n_rb + 1);
    griddep_launch_dependents();
    griddep_wait();
    const int t = __ldcg(tp) + local;
    // slots past the end of a head's list (lists of different lengths per layout head) are unused
    const int hb = t < __ldcg(tp + sc.n_rb) ? tinfo_half(__ldcg(sc.tinfo + t)) : 0;
    if (hb == 0) return;
    // LS: scores S (plain GEMM1 output, in pbuf) -> X' (xprime);  GS: X' -> Y = X' r' (pbuf)
    const uint8_t* src = (const uint8_t*)(LS ? p.pbuf : p.xprime) + slot * (int64_t)XB;
    uint8_t* dst = (uint8_t*)(LS ? p.xprime : p.pbuf) + slot * (int64_t)XB;
    if (threadIdx.x == 0) {
        mbar_init(&bar, 1);
        fence_mbar_init();
        mbar_arrive_expect_tx(&bar, XB);
        bulk_load(tile, src, XB, &bar);
    }
    __syncthreads();
    mbar_wait(&bar, 0);
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if ((hb >> (warp / 2)) & 1) {
        const float l2e = 1.4426950408889634f;
        const bool bf = p.in_dtype == DT_BF16;
        for (int rr = 0; rr < 32; ++rr) {
            const int r = warp * 32 + rr;
            const uint32_t base = smem_u32(tile) + r * 128 + lane * 4;
            float2 f[NP];
#pragma unroll
            for (int c = 0; c < NP; ++c) f[c] = unpack_f16(lds_u32(base + c * (kRowBlock * 128)));
            if (LS) {  // LS: m' = row max of the tile, X' = e^{x - m'}, d' = sum X'
                float mx = -INFINITY;
#pragma unroll
                for (int c = 0; c < NP; ++c) mx = fmaxf(mx, fmaxf(f[c].x, f[c].y));
                for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
                const float neg = (mx == -INFINITY) ? 0.f : -mx * l2e;
                float sum = 0.f;
#pragma unroll
                for (int c = 0; c < NP; ++c) {
                    const float y0 = ex2(fmaf(f[c].x, l2e, neg)), y1 = ex2(fmaf(f[c].y, l2e, neg));
                    sum += y0 + y1;
                    sts_u32(base + c * (kRowBlock * 128), pack_f16(y0, y1));
                }
                for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
                if (lane == 0) {
                    p.mprime[slot * kRowBlock + r] = mx;  // scores already carry the scale: natural-log units
                    p.dprime[slot * kRowBlock + r] = sum;
                }
            } else {  // GS: element-wise scaling by the row's reconstruction factor
                const float rr_ = __ldcg(p.rprime + slot * kRowBlock + r);
#pragma unroll
                for (int c = 0; c < NP; ++c)
                    sts_u32(base + c * (kRowBlock * 128),
                            bf ? pack_bf16(f[c].x * rr_, f[c].y * rr_) : pack_f16(f[c].x * rr_, f[c].y * rr_));
            }
        }
    }
    fence_proxy_async_smem();
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int h = 0; h < 2; ++h) {
            if (!((hb >> h) & 1)) continue;
            for (int c = 0; c < NP; ++c)
                bulk_store(dst + c * (kRowBlock * 128) + h * (kHalf * 128), tile + c * (kRowBlock * 128) + h * (kHalf * 128),
                           kHalf * 128);
        }
        bulk_commit();
        bulk_wait_read0();
    }
}

cudaError_t launch_gemm1(const Params& p, bool ls, cudaStream_t st, int64_t* nl);
cudaError_t launch_gemm2(const Params& p, int mode, cudaStream_t st, int64_t* nl);

template <int T>
cudaError_t launch_sd_t(const Params& p, cudaStream_t st, int64_t* nl)
{
    const unsigned blocks = (unsigned)((int64_t)p.B * p.H * p.sc.slots_per_head);
    cudaError_t e = cudaSuccess;
    if (p.stages & 2) {
        if ((e = launch_pdl(sd_tile_kernel<T, true>, dim3(blocks), dim3(128), 0, st, nl, p)) != cudaSuccess) return e;
        if ((e = launch_ir(p, st, nl)) != cudaSuccess) return e;
        if ((e = launch_pdl(sd_tile_kernel<T, false>, dim3(blocks), dim3(128), 0, st, nl, p)) != cudaSuccess) return e;
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
