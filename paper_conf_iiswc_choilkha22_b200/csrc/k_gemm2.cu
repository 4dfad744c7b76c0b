// k_gemm2.cu -- GS + GEMM2 kernel and launchers; the device code is in g2_body.cuh.
#include "g2_body.cuh"

namespace sr {

using namespace ptx;

#ifdef SR_DIAG_WAITS
}  // namespace sr
extern "C" int sr_diag_read_g2(unsigned long long* out)  // copies [32 warps][kDW + 1] and resets (diagnostic build)
{
    if (cudaMemcpyFromSymbol(out, sr::g_diag_g2, sizeof(sr::g_diag_g2)) != cudaSuccess) return 1;
    static unsigned long long zero[32 * (sr::kDW + 1)];
    return cudaMemcpyToSymbol(sr::g_diag_g2, zero, sizeof(zero)) != cudaSuccess;
}
namespace sr {
#endif

template <int D, int T, bool GS, bool FI, bool RS>
__global__ void __launch_bounds__(G2<D, T>::THREADS, 1) tc_gemm2(const __grid_constant__ CUtensorMap tmV, const Params p)
{
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint32_t* tmem_ptr = (uint32_t*)(smem + G2<D, T>::OFF_TPTR);
    const int warp = warp_uniform(), lane = threadIdx.x % 32;
    if (threadIdx.x == 0) g2_init<D, T, GS, FI, RS>(smem);
    if (warp == 3 && lane == 0) prefetch_tmap(&tmV);
    if (warp == 2) tmem_alloc(tmem_ptr, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_ptr;
    // PDL: the prologue above overlapped the previous kernel's tail; let the next kernel start its
    // own prologue, then wait for our producer kernel's results before touching them
    griddep_launch_dependents();
    griddep_wait();
    g2_roles<D, T, GS, FI, RS>(tmV, p, p.sc, smem, tmem_base, __ldca(p.sc.cta_ptr + blockIdx.x),
                               __ldca(p.sc.cta_ptr + blockIdx.x + 1));
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

// ----------------------------------------------------------------------------- launchers

cudaError_t make_tmap_2d(CUtensorMap* m, const void* base, int64_t rows, int D, int box_rows, int dtype);
int num_sms();

template <int D, int T, bool GS, bool FI, bool RS>
cudaError_t launch_g2_t(const Params& p, cudaStream_t st, int64_t* nl)
{
    using C = G2<D, T>;
    CUtensorMap tv;
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    cudaError_t e;
    if ((e = make_tmap_2d(&tv, p.v, rows, D, T, p.in_dtype)) != cudaSuccess) return e;
    auto kern = tc_gemm2<D, T, GS, FI, RS>;
    if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM)) != cudaSuccess) return e;
    const int grid = p.sc.n_cta;  // one persistent CTA per SM, items assigned by host LPT
    return launch_pdl(kern, dim3(grid), dim3(C::THREADS), C::SMEM, st, nl, tv, p);
}

template <int D, int T>
cudaError_t launch_g2_dt(const Params& p, int mode, cudaStream_t st, int64_t* nl)
{
    if (mode == 0) return launch_g2_t<D, T, false, false, false>(p, st, nl);
    if (mode == 1) return launch_g2_t<D, T, true, false, false>(p, st, nl);
    if (mode == 2) return launch_g2_t<D, T, true, true, false>(p, st, nl);
    return launch_g2_t<D, T, true, true, true>(p, st, nl);
}

// mode: 0 = unfused baseline (P . V), 1 = GS + GEMM2 (r' from the IR kernel), 2 = IR + GS + GEMM2,
// 3 = GS + GEMM2 on the (m, 1/d) rows GEMM1 merged
cudaError_t launch_gemm2(const Params& p, int mode, cudaStream_t st, int64_t* nl)
{
    if (p.D == 64) return p.T == 64 ? launch_g2_dt<64, 64>(p, mode, st, nl) : launch_g2_dt<64, 128>(p, mode, st, nl);
    return p.T == 64 ? launch_g2_dt<128, 64>(p, mode, st, nl) : launch_g2_dt<128, 128>(p, mode, st, nl);
}

}  // namespace sr
