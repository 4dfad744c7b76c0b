// k_ir.cu -- the IR (inter-sub-vector reduction) sub-layer.
//
// Per query row:  m = max_k m'_k,   d = sum_k e^{m'_k - m} d'_k,   r'_k = e^{m'_k - m} / d.
// One thread per row.  The statistics are stored [slot][128 rows], so the 32 threads of a warp
// (32 consecutive rows of one row-block) read and write 128 contiguous bytes per tile: fully
// coalesced.  The kernel is HBM/latency bound: 8 bytes read + 4 bytes written per (row, tile),
// i.e. 1/T of the attention-matrix traffic.  It cannot be fused into GEMM1
// (m, d need every tile of the row) -- the paper's design keeps it standalone.
#include "sr_internal.h"

namespace sr {

__global__ void __launch_bounds__(256) ir_kernel(Params p)
{
    const int64_t row = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t n_rows = (int64_t)p.B * p.H * p.S;
    if (row >= n_rows) return;
    const int g = (int)(row / p.S);
    const int i = (int)(row % p.S);
    const int rb = i / kRowBlock, lane = i % kRowBlock, half = lane / kHalf;
    const DevSched& sc = p.sc;
    const int lh = lh_of(sc, g, p.H);
    const int32_t* tp = sc.tp + (size_t)lh * (sc.n_rb + 1);
    const int t0 = tp[rb], t1 = tp[rb + 1], base = tp[0];
    const int64_t slot0 = (int64_t)g * sc.slots_per_head - base;

    float m = -INFINITY;
    for (int t = t0; t < t1; ++t) {
        if (!((tinfo_half(__ldg(sc.tinfo + t)) >> half) & 1)) continue;
        m = fmaxf(m, __ldg(p.mprime + (slot0 + t) * kRowBlock + lane));
    }
    float d = 0.f;
    if (m != -INFINITY) {
        for (int t = t0; t < t1; ++t) {
            if (!((tinfo_half(__ldg(sc.tinfo + t)) >> half) & 1)) continue;
            const float mk = __ldg(p.mprime + (slot0 + t) * kRowBlock + lane);
            if (mk != -INFINITY) d += expf(mk - m) * __ldg(p.dprime + (slot0 + t) * kRowBlock + lane);
        }
    }
    const float inv_d = d > 0.f ? 1.f / d : 0.f;
    for (int t = t0; t < t1; ++t) {
        float r = 0.f;
        if ((tinfo_half(__ldg(sc.tinfo + t)) >> half) & 1) {
            const float mk = __ldg(p.mprime + (slot0 + t) * kRowBlock + lane);
            if (mk != -INFINITY) r = expf(mk - m) * inv_d;
        }
        p.rprime[(slot0 + t) * kRowBlock + lane] = r;
    }
}

cudaError_t launch_ir(const Params& p, cudaStream_t st, int64_t* nlaunch)
{
    const int64_t n_rows = (int64_t)p.B * p.H * p.S;
    const int threads = 256;
    const int64_t blocks = (n_rows + threads - 1) / threads;
    ir_kernel<<<(unsigned)blocks, threads, 0, st>>>(p);
    ++*nlaunch;
    return cudaGetLastError();
}

}  // namespace sr
