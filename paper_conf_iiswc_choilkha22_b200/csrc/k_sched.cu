// k_sched.cu -- stream-ordered upload of a call's tile schedule into the caller's workspace.
//
// The schedule (item lists, tile lists, per-CTA ranges; abi.cu) is derived on the host from the mask
// descriptor of the call (the mask is an input of every call).  It lives in the
// caller-owned workspace (region off_sched, include/sr_mha.h), never in library-owned device
// memory, and reaches it through the KERNEL PARAMETERS of this copy kernel: the words travel inside
// the launch itself, so
//   - nothing is allocated and nothing synchronises (no cudaMalloc, no blocking cudaMemcpy),
//   - the upload is a plain stream-ordered kernel node, capturable in a CUDA graph: a graph replay
//     re-writes exactly the schedule its call captured, whatever other calls did in between,
//   - there is no host buffer whose lifetime a pending copy or a graph would depend on.
// A launch carries up to kChunkVec 16-B words (~31 KB of parameter space; the limit is 32764 B);
// larger schedules take several launches.  Each launch is PDL-chained like every sr kernel: it may
// start while the previous kernel drains but writes only after griddepcontrol.wait (that kernel may
// still be reading the previous call's schedule from the same workspace), and the kernel that
// consumes the schedule waits for this one the same way.
#include <cstring>

#include "ptx.cuh"
#include "sr_internal.h"

namespace sr {

namespace {

constexpr int kMaxSeg = 8;
constexpr int kChunkVec = 1984;  // 16-B words per launch (31,744 B)

struct SchedChunk {
    int32_t n_seg;
    int32_t dst[kMaxSeg];  // destination offset of each segment, in 16-B words from the region base
    int32_t len[kMaxSeg];  // segment length in 16-B words; segments are packed back to back in data
    int4 data[kChunkVec];
};
static_assert(sizeof(SchedChunk) + sizeof(void*) <= 32764, "kernel parameter space");

__global__ void __launch_bounds__(256) sched_upload(int4* __restrict__ region, const __grid_constant__ SchedChunk c)
{
    ptx::griddep_launch_dependents();
    // one 16-B word per thread (the grid covers the chunk): every load in flight at once.  The
    // payload is read through its generic address (coalesced; indexed constant-bank loads with a
    // different address per lane would serialise).
    const int4* data;
    asm("mov.b64 %0, %1;" : "=l"(data) : "l"(&c.data[0]));  // opaque to the compiler: stays generic
    int i = blockIdx.x * blockDim.x + threadIdx.x, s = 0;
    while (s < c.n_seg && i >= c.len[s]) i -= c.len[s++];
    int src = 0;
    for (int k = 0; k < s; ++k) src += c.len[k];
    const int4 v = s < c.n_seg ? data[src + i] : make_int4(0, 0, 0, 0);
    ptx::griddep_wait();  // the previous kernel may still read the region
    if (s < c.n_seg) region[c.dst[s] + i] = v;
}

}  // namespace

cudaError_t launch_sched_upload(void* region, const int32_t* words, const size_t* seg_off, const size_t* seg_len,
                                int n_seg, cudaStream_t st, int64_t* nl)
{
    thread_local SchedChunk c;  // 31 KB staging of the launch parameters (copied at launch)
    c.n_seg = 0;
    int fill = 0;
    cudaError_t e = cudaSuccess;
    auto flush = [&]() -> cudaError_t {
        if (c.n_seg == 0) return cudaSuccess;
        cudaError_t r = launch_pdl(sched_upload, dim3((unsigned)((fill + 255) / 256)), dim3(256), 0, st, nl,
                                   (int4*)region, c);
        c.n_seg = 0;
        fill = 0;
        return r;
    };
    for (int s = 0; s < n_seg; ++s) {
        // offsets and lengths are in int32 words, multiples of 4 (abi.cu pads every group)
        size_t off = seg_off[s] / 4, left = seg_len[s] / 4;
        while (left > 0) {
            if (c.n_seg == kMaxSeg || fill == kChunkVec)
                if ((e = flush()) != cudaSuccess) return e;
            const size_t take = left < (size_t)(kChunkVec - fill) ? left : (size_t)(kChunkVec - fill);
            c.dst[c.n_seg] = (int32_t)off;
            c.len[c.n_seg] = (int32_t)take;
            memcpy(&c.data[fill], words + off * 4, take * 16);
            ++c.n_seg;
            fill += (int)take;
            off += take;
            left -= take;
        }
    }
    return flush();
}

}  // namespace sr
