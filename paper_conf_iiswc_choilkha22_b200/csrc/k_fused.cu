// k_fused.cu -- the recomposed layer in ONE launch (variant SR_ONE_KERNEL).
//
// A GEMM1 CTA owns whole query rows (every key tile of its row-blocks, IR merged in GEMM1), so the
// GS + GEMM2 work of those rows depends on nothing another CTA computes.  Each persistent CTA
// therefore runs
//   phase 1  GEMM1 + LS + IR over its row-blocks (g1_body.cuh): X' tiles and m' to the
//            workspace, per-row (m, d) partials to rowstat
//   phase 2  GS + GEMM2 over the same row-blocks (g2_body.cuh), reading back the X' it wrote
//            (the attention matrix still crosses memory once each way, L171-L173)
// separated by a CTA barrier instead of a kernel boundary: no second launch and no grid-wide wait
// for the slowest GEMM1 CTA (measured, one B200: C2 27.6 -> 24.6 us, C5 80.9 -> 72.6 us).
// Cutting each CTA's items into L2-sized chunks (one launch per chunk, X' kept with evict_last)
// was slower on C3-C5 (grid-wide tails per chunk); a chunk loop inside the kernel makes ptxas
// spill the setmaxnreg-rebalanced epilogues.  X' stores stay evict_first.
// T = 64 (reading R3): the SPLIT GEMM1 epilogue (four warpgroups, 104 registers) leaves the
// register budget of a 640-thread CTA that GEMM2's 16 warps can reuse in phase 2.
#include "g1_body.cuh"
#include "g2_body.cuh"

namespace sr {

using namespace ptx;

#ifdef SR_DIAG_PHASES
// diagnostic build: per CTA, %globaltimer (ns) at kernel start, after the prologue, after phase 1,
// after phase 2, plus the CTA's item count (read with sr_diag_read_phases)
__device__ unsigned long long g_diag_phases[1024 * 8];
__device__ __forceinline__ unsigned long long gtimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#define PH_MARK(i) do { if (threadIdx.x == 0) g_diag_phases[blockIdx.x * 8 + (i)] = gtimer(); } while (0)
#else
#define PH_MARK(i)
#endif

template <int D, bool PAIR>
__global__ void __launch_bounds__(640, 1)
    tc_fused(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
             const __grid_constant__ CUtensorMap tmV, const Params p)
{
    using C1 = G1<D, 64, PAIR>;
    using C2 = G2<D, 64>;
    static_assert(C1::THREADS == 640 && (C2::THREADS <= 640 || SR_G2_NGS != 8), "warp budget");
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    uint32_t* tmem_ptr = (uint32_t*)(smem + C1::OFF_TPTR);
    const int warp = warp_uniform(), lane = threadIdx.x % 32;
    const DevSched& sc = p.sc;  // the schedule the call uploaded into its workspace (k_sched.cu)
    PH_MARK(0);
    if (threadIdx.x == 0) g1_init<D, 64, true, PAIR, true>(smem);
    if (warp == 0 && lane == 0) { prefetch_tmap(&tmQ); prefetch_tmap(&tmK); prefetch_tmap(&tmV); }
    if (warp == 2) tmem_alloc(tmem_ptr, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_ptr;
    griddep_launch_dependents();
    griddep_wait();

    // phase 2's row-blocks (with PAIR the host pointed cta_ptr / item_desc at the pair assignment
    // unrolled into row-blocks, so both phases cover the same rows)
    const int it_begin = __ldca(sc.cta_ptr + blockIdx.x), it_end = __ldca(sc.cta_ptr + blockIdx.x + 1);
    // phase 2 applies Global Scaling accumulator-side for fp16 (X' and V share the MMA type; see
    // g2_body.cuh AS) unless p.gs_prologue; bf16 V needs the prologue form (Y rounded to bf16)
    // (D = 64: the scaling warps hold D/2 fp32 of O each within the 96-register phase-2 budget)
    const bool as = D == 64 && p.in_dtype == DT_F16 && !p.gs_prologue;
    PH_MARK(1);
    // ---- phase 1: GEMM1 + LS + IR over the CTA's row-blocks (all 20 warps)
    if constexpr (PAIR)
        g1_roles<D, 64, true, true, true>(tmQ, tmK, p, sc, smem, tmem_base, __ldca(sc.pcta_ptr + blockIdx.x),
                                          __ldca(sc.pcta_ptr + blockIdx.x + 1));
    else
        g1_roles<D, 64, true, false, true>(tmQ, tmK, p, sc, smem, tmem_base, it_begin, it_end);
    // back to the launch split (phase 1 leaves warps 0-3 at 64 registers, the epilogue at 104)
    if (warp < 4) reg_alloc<96>();
    else reg_dealloc<96>();
    // the X' bulk stores are complete (each storing lane ended with wait_group 0); m' and rowstat
    // were written through the generic proxy and are read back by bulk copies / loads below
    fence_proxy_async_global();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    PH_MARK(2);
    if (threadIdx.x == 0) {
        uint64_t* b1 = (uint64_t*)(smem + C1::OFF_BAR);
        for (int i = 0; i < C1::NBAR; ++i) mbar_inval(&b1[i]);
        if (as) g2_init<D, 64, true, true, true, D == 64>(smem);
        else g2_init<D, 64, true, true, true>(smem);
    }
    __syncthreads();
    // ---- phase 2: GS + GEMM2 over the same row-blocks (warps 0-15; 16-19 idle)
    if constexpr (D == 64) {
        if (as) g2_roles<D, 64, true, true, true, true>(tmV, p, sc, smem, tmem_base, it_begin, it_end);
        else g2_roles<D, 64, true, true, true>(tmV, p, sc, smem, tmem_base, it_begin, it_end);
    } else {
        g2_roles<D, 64, true, true, true>(tmV, p, sc, smem, tmem_base, it_begin, it_end);
    }
    tc_fence_before();
    __syncthreads();
    PH_MARK(3);
#ifdef SR_DIAG_PHASES
    if (threadIdx.x == 0) {
        g_diag_phases[blockIdx.x * 8 + 4] = it_end - it_begin;
        unsigned long long nt = 0;  // the CTA's listed tiles and its SM
        for (int it = it_begin; it < it_end; ++it) {
            const int4 d = __ldca(sc.item_desc + it);
            nt += d.z - d.y;
        }
        unsigned smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        g_diag_phases[blockIdx.x * 8 + 5] = nt;
        g_diag_phases[blockIdx.x * 8 + 6] = smid;
    }
#endif
    if (warp == 2) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

cudaError_t make_tmap_2d(CUtensorMap* m, const void* base, int64_t rows, int D, int box_rows, int dtype);

template <int D>
cudaError_t launch_one_d(const Params& p, cudaStream_t st, int64_t* nl)
{
    CUtensorMap tq, tk, tv;
    const int64_t rows = (int64_t)p.B * p.H * p.S;
    cudaError_t e;
    if ((e = make_tmap_2d(&tq, p.q, rows, D, kRowBlock, p.in_dtype)) != cudaSuccess) return e;
    if ((e = make_tmap_2d(&tk, p.k, rows, D, 64, p.in_dtype)) != cudaSuccess) return e;
    if ((e = make_tmap_2d(&tv, p.v, rows, D, 64, p.in_dtype)) != cudaSuccess) return e;
    constexpr int s0 = G1<D, 64, false>::SMEM > G2<D, 64>::SMEM ? G1<D, 64, false>::SMEM : G2<D, 64>::SMEM;
    constexpr int s1 = G1<D, 64, true>::SMEM > G2<D, 64>::SMEM ? G1<D, 64, true>::SMEM : G2<D, 64>::SMEM;
    auto kern = p.g1_pair ? tc_fused<D, true> : tc_fused<D, false>;
    const int smem = p.g1_pair ? s1 : s0;
    if ((e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
    return launch_pdl(kern, dim3(p.sc.n_cta), dim3(640), smem, st, nl, tq, tk, tv, p);
}

cudaError_t launch_tc_one(const Params& p, cudaStream_t st, int64_t* nl)
{
    if (p.T != 64) return cudaErrorInvalidValue;
    return p.D == 64 ? launch_one_d<64>(p, st, nl) : launch_one_d<128>(p, st, nl);
}

}  // namespace sr

#ifdef SR_DIAG_WAITS
// the fused kernel's phase-1 / phase-2 wait counters (this translation unit's copies)
extern "C" int sr_diag_read_fused(int phase, unsigned long long* out)  // [32][kDW + 1], reset after read
{
    void* sym = nullptr;
    if (cudaGetSymbolAddress(&sym, phase == 1 ? sr::g_diag_g1 : sr::g_diag_g2) != cudaSuccess) return 1;
    const size_t n = sizeof(sr::g_diag_g1);
    if (cudaMemcpy(out, sym, n, cudaMemcpyDeviceToHost) != cudaSuccess) return 1;
    return cudaMemset(sym, 0, n) != cudaSuccess;
}
#endif

#ifdef SR_DIAG_PHASES
extern "C" int sr_diag_read_phases(unsigned long long* out)  // [1024][8] (diagnostic build)
{
    return cudaMemcpyFromSymbol(out, sr::g_diag_phases, sizeof(sr::g_diag_phases)) != cudaSuccess;
}
#endif
