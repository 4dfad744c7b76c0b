// k_conc.cu -- the recomposed layer with GEMM1 and GEMM2 running CONCURRENTLY in one persistent CTA
// per SM (variant SR_CONCURRENT).
//
// The one-launch kernel (k_fused.cu) runs its CTA's items through phase 1 (GEMM1 + LS + IR) and only
// then through phase 2 (GS + GEMM2): the two phases never overlap on an SM, and all but the last
// items' X' has left the L2 by the time phase 2 reads it back.  Here both role sets are resident at
// once, on disjoint warps, shared memory and TMEM of the same CTA:
//
//   warps  0-3   GEMM1 control: TMA (Q, K), MMA issue, the two IR warps
//   warps  4-11  GEMM1 + LS epilogue: two warpgroups, alternate 64-key macro tiles (L131-L145)
//   warps 12-15  GEMM2 control: X' + m' producer, MMA issue, row statistics, V producer
//   warps 16-23  GS: Y = X' r' into the TMEM A operand (L151)
//   warps 24-27  GEMM2 epilogue: O rows to global
//
// GEMM2 takes an item (head, row-block) over as soon as GEMM1 has finished it: every GEMM1 epilogue
// warp announces an item once its X' bulk stores and m' of that item are complete, the IR warps once
// the item's row statistics (m, d) are written (mbarrier ring item_done); GEMM2's producers wait for
// that, and GEMM1 never starts an item more than kConcNI items ahead of GEMM2 (ring item_free).  X'
// is still written to HBM and read back (the matrix crosses memory once each way), but
// GEMM2 reads it while it is still in L2, and the two GEMMs' different bottlenecks (GEMM1: MUFU
// exponentials and the X' store stream; GEMM2: the GS pass and the X' / V load streams) overlap.
//
// Resources (D = 128): TMEM 128 columns for GEMM1's two 128 x 64 fp32 accumulators + 384 for GEMM2
// (two O accumulators, four A buffers); shared memory split Conc<D>::B1 / B2; 896 threads at 72
// registers rebalanced per warpgroup with setmaxnreg (48 / 104 / 104 / 40 / 72 / 72 / 64: the
// budget balances exactly, 28 warps x 72).
#include "g1_body.cuh"
#include "g2_body.cuh"

namespace sr {

using namespace ptx;

#if SR_G2_NGS == 8  // the warp layout below assumes GEMM2's default 8 GS warps (experiment builds skip it)
constexpr int kConcThreads = 896;
constexpr int kConcT1 = 128;         // GEMM1 TMEM columns

template <int D>
struct Conc {
    // shared-memory budgets: D = 128: GEMM1 Q, 3 K stages, 2 staging tiles | GEMM2 4 X' + 2 V stages;
    // D = 64: GEMM1 2 Q, 3 K stages, 2 x 2 staging tiles | GEMM2 4 X' + 2 V stages
    static constexpr int B1 = D == 128 ? 118 * 1024 : 126 * 1024;
    static constexpr int B2 = D == 128 ? 104 * 1024 : 100 * 1024;
    using C1 = G1<D, 64, false, 64, B1>;
    using C2 = G2<D, 64, 64, B2, 512 - kConcT1>;
    static constexpr int OFF2 = (C1::OFF_TPTR + 16 + 1023) / 1024 * 1024;  // GEMM2's region (1 KB aligned)
    static constexpr int OFF_IBAR = OFF2 + C2::OFF_TPTR + 16;
    static constexpr int SMEM = OFF_IBAR + 2 * kConcNI * 8 + 1024;  // + alignment slack
    static_assert(SMEM <= kSmemMax, "smem budget");
    static_assert(C1::THREADS == 384 && C2::THREADS == 512, "warp layout");
};

template <int D>
__global__ void __launch_bounds__(kConcThreads, 1)
    tc_conc(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
            const __grid_constant__ CUtensorMap tmV, const Params p)
{
    using K = Conc<D>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint8_t* smem2 = smem + K::OFF2;
    uint64_t* ibar = (uint64_t*)(smem + K::OFF_IBAR);
    uint32_t* tmem_ptr = (uint32_t*)(smem + K::C1::OFF_TPTR);
    const int warp = warp_uniform(), lane = threadIdx.x % 32;
    const DevSched& sc = p.sc;
    if (threadIdx.x == 0) {
        g1_init<D, 64, true, false, true, 64, K::B1>(smem);
        g2_init<D, 64, true, true, true, false, 64, K::B2, 512 - kConcT1>(smem2);
        // item_done: 8 GEMM1 epilogue warps + 2 IR warps; item_free: GEMM2's X' producer + statistics warp
        for (int i = 0; i < kConcNI; ++i) { mbar_init(&ibar[i], 10); mbar_init(&ibar[kConcNI + i], 2); }
        fence_mbar_init();
    }
    if (warp == 0 && lane == 0) { prefetch_tmap(&tmQ); prefetch_tmap(&tmK); prefetch_tmap(&tmV); }
    if (warp == 2) tmem_alloc(tmem_ptr, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_ptr;
    griddep_launch_dependents();
    griddep_wait();
    const int it_begin = __ldca(sc.cta_ptr + blockIdx.x), it_end = __ldca(sc.cta_ptr + blockIdx.x + 1);
    // each role group under its own register budget (setmaxnreg dominates the group's code)
    if (warp < 4) {
        reg_dealloc<48>();
        g1_roles<D, 64, true, false, true, false, 64, K::B1, true, 1>(tmQ, tmK, p, sc, smem, tmem_base, it_begin,
                                                                        it_end, ibar);
    } else if (warp < 12) {
        reg_alloc<104>();
        g1_roles<D, 64, true, false, true, false, 64, K::B1, true, 2>(tmQ, tmK, p, sc, smem, tmem_base, it_begin,
                                                                        it_end, ibar);
    } else if (warp < 16) {
        reg_dealloc<40>();
        g2_roles<D, 64, true, true, true, false, 64, K::B2, 512 - kConcT1, 12, true, 1>(
            tmV, p, sc, smem2, tmem_base + kConcT1, it_begin, it_end, ibar);
    } else if (warp < 24) {
        g2_roles<D, 64, true, true, true, false, 64, K::B2, 512 - kConcT1, 12, true, 2>(
            tmV, p, sc, smem2, tmem_base + kConcT1, it_begin, it_end, ibar);
    } else {
        reg_dealloc<64>();
        g2_roles<D, 64, true, true, true, false, 64, K::B2, 512 - kConcT1, 12, true, 4>(
            tmV, p, sc, smem2, tmem_base + kConcT1, it_begin, it_end, ibar);
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

cudaError_t make_tmap_2d(CUtensorMap* m, const void* base, int64_t rows, int D, int box_rows, int dtype);

template <int D>
cudaError_t launch_conc_d(const Params& p, cudaStream_t st, int64_t* nl)
{
    CUtensorMap tq, tk, tv;
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    cudaError_t e;
    if ((e = make_tmap_2d(&tq, p.q, rows, D, kRowBlock, p.in_dtype)) != cudaSuccess) return e;
    if ((e = make_tmap_2d(&tk, p.k, rows, D, 64, p.in_dtype)) != cudaSuccess) return e;
    if ((e = make_tmap_2d(&tv, p.v, rows, D, 64, p.in_dtype)) != cudaSuccess) return e;
    auto kern = tc_conc<D>;
    constexpr int smem = Conc<D>::SMEM;
    if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
    return launch_pdl(kern, dim3(p.sc.n_cta), dim3(kConcThreads), smem, st, nl, tq, tk, tv, p);
}

cudaError_t launch_tc_conc(const Params& p, cudaStream_t st, int64_t* nl)
{
    if (p.T != 64 || p.in_dtype == DT_F32 || p.g1_pair) return cudaErrorInvalidValue;
    return p.D == 128 ? launch_conc_d<128>(p, st, nl) : launch_conc_d<64>(p, st, nl);
}
#else
cudaError_t launch_tc_conc(const Params&, cudaStream_t, int64_t*) { return cudaErrorNotSupported; }
#endif

}  // namespace sr

#ifdef SR_DIAG_WAITS
// the concurrent kernel's wait counters (this translation unit's copies): which = 1 GEMM1 roles
// (warps 0-11), 2 GEMM2 roles (warps 12-27); [32][kDW + 1], reset after read
extern "C" int sr_diag_read_conc(int which, unsigned long long* out)
{
    void* sym = nullptr;
    if (cudaGetSymbolAddress(&sym, which == 1 ? sr::g_diag_g1 : sr::g_diag_g2) != cudaSuccess) return 1;
    const size_t n = sizeof(sr::g_diag_g1);
    if (cudaMemcpy(out, sym, n, cudaMemcpyDeviceToHost) != cudaSuccess) return 1;
    return cudaMemset(sym, 0, n) != cudaSuccess;
}
#endif
