// k_g1.cu -- GEMM1 + LS (+ IR) kernel and launchers; the device code is in g1_body.cuh.
#include "g1_body.cuh"

namespace sr {

using namespace ptx;

#ifdef SR_DIAG_WAITS
}  // namespace sr
extern "C" int sr_diag_read_g1(unsigned long long* out)  // copies [32 warps][kDW + 1] and resets (diagnostic build)
{
    if (cudaMemcpyFromSymbol(out, sr::g_diag_g1, sizeof(sr::g_diag_g1)) != cudaSuccess) return 1;
    static unsigned long long zero[32 * (sr::kDW + 1)];
    return cudaMemcpyToSymbol(sr::g_diag_g1, zero, sizeof(zero)) != cudaSuccess;
}
namespace sr {
#endif

template <int D, int T, bool LS, bool PAIR, bool IRT>
__global__ void __launch_bounds__(T == 64 ? 640 : 384, 1)
    tc_gemm1(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK, const Params p)
{
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint32_t* tmem_ptr = (uint32_t*)(smem + G1<D, T, PAIR>::OFF_TPTR);
    const int warp = warp_uniform(), lane = threadIdx.x % 32;
    if (threadIdx.x == 0) g1_init<D, T, LS, PAIR, IRT>(smem);
    if (warp == 0 && lane == 0) { prefetch_tmap(&tmQ); prefetch_tmap(&tmK); }
    if (warp == 2) tmem_alloc(tmem_ptr, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_ptr;
    // PDL: the prologue above overlapped the previous kernel's tail; let the next kernel start its
    // own prologue, then wait for our producer kernel's results before touching them
    griddep_launch_dependents();
    griddep_wait();
    // this CTA's items (row-blocks, or pairs of row-blocks): a contiguous range of the host's
    // longest-processing-time assignment
    const int32_t* cptr = PAIR ? p.sc.pcta_ptr : p.sc.cta_ptr;
    g1_roles<D, T, LS, PAIR, IRT>(tmQ, tmK, p, p.sc, smem, tmem_base, __ldca(cptr + blockIdx.x), __ldca(cptr + blockIdx.x + 1));
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

template <int D, int T, bool LS, bool PAIR, bool IRT>
cudaError_t launch_g1_t(const Params& p, cudaStream_t st, int64_t* nl)
{
    using C = G1<D, T, PAIR>;
    CUtensorMap tq, tk;
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    cudaError_t e;
    if ((e = make_tmap_2d(&tq, p.q, rows, D, kRowBlock, p.in_dtype)) != cudaSuccess) return e;
    if ((e = make_tmap_2d(&tk, p.k, rows, D, T, p.in_dtype)) != cudaSuccess) return e;
    auto kern = tc_gemm1<D, T, LS, PAIR, IRT>;
    if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM)) != cudaSuccess) return e;
    const int grid = PAIR ? p.sc.n_pcta : p.sc.n_cta;  // one persistent CTA per SM, host LPT items
    return launch_pdl(kern, dim3(grid), dim3(C::THREADS), C::SMEM, st, nl, tq, tk, p);
}

template <int D, int T, bool LS>
cudaError_t launch_g1_p(const Params& p, cudaStream_t st, int64_t* nl)
{
    if (LS && p.ir_mode == IR_IN_GEMM1)
        return p.g1_pair ? launch_g1_t<D, T, LS, true, LS>(p, st, nl) : launch_g1_t<D, T, LS, false, LS>(p, st, nl);
    return p.g1_pair ? launch_g1_t<D, T, LS, true, false>(p, st, nl) : launch_g1_t<D, T, LS, false, false>(p, st, nl);
}

cudaError_t launch_gemm1(const Params& p, bool ls, cudaStream_t st, int64_t* nl)
{
    if (p.D == 64) {
        if (p.T == 64) return ls ? launch_g1_p<64, 64, true>(p, st, nl) : launch_g1_p<64, 64, false>(p, st, nl);
        return ls ? launch_g1_p<64, 128, true>(p, st, nl) : launch_g1_p<64, 128, false>(p, st, nl);
    }
    if (p.T == 64) return ls ? launch_g1_p<128, 64, true>(p, st, nl) : launch_g1_p<128, 64, false>(p, st, nl);
    return ls ? launch_g1_p<128, 128, true>(p, st, nl) : launch_g1_p<128, 128, false>(p, st, nl);
}

}  // namespace sr
