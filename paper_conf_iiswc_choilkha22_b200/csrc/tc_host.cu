// tc_host.cu -- host side of the tensor-core path: TMA descriptors (cuTensorMapEncodeTiled via the
// runtime's driver entry point, no libcuda link), SM count, and the three-kernel launch sequences
// of the recomposed chain (GEMM1+LS -> IR -> GS+GEMM2) and of the unfused
// baseline (GEMM1 -> row softmax -> GEMM2, L171).
#include <cuda.h>

#include <mutex>

#include "sr_internal.h"

namespace sr {

cudaError_t launch_gemm1(const Params& p, bool ls, cudaStream_t st, int64_t* nl);
cudaError_t launch_gemm2(const Params& p, int mode, cudaStream_t st, int64_t* nl);
cudaError_t launch_softmax(const Params& p, cudaStream_t st, int64_t* nl);

namespace {
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn encode_fn()
{
    static EncodeTiledFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeTiledFn)f;
    });
    return fn;
}
}  // namespace

// [rows][D] 16-bit row-major tensor, box {64 cols = 128 B, box_rows}, 128-B swizzle
cudaError_t make_tmap_2d(CUtensorMap* m, const void* base, int64_t rows, int D, int box_rows, int dtype)
{
    EncodeTiledFn fn = encode_fn();
    if (!fn) return cudaErrorNotSupported;
    cuuint64_t dims[2] = {(cuuint64_t)D, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)D * 2};
    cuuint32_t box[2] = {64, (cuuint32_t)box_rows};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = fn(m, dtype == DT_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2,
                    const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

int num_sms()
{
    int dev = 0, n = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    return n;
}

cudaError_t launch_tc_fused(const Params& p, cudaStream_t st, int64_t* nl)
{
    cudaError_t e = cudaSuccess;
    if ((p.stages & 1) && (e = launch_gemm1(p, true, st, nl)) != cudaSuccess) return e;
    // the IR sub-layer: its own kernel (SR_IR_KERNEL, the paper's layout), folded into GEMM2 (SR_FUSE_IR), or
    // merged inside GEMM1 (the default, GEMM2 then only reads each row's (m, 1/d))
    if (p.ir_mode == IR_KERNEL && (p.stages & 2) && (e = launch_ir(p, st, nl)) != cudaSuccess) return e;
    if (p.stages & 4) e = launch_gemm2(p, p.ir_mode == IR_KERNEL ? 1 : (p.ir_mode == IR_IN_GEMM2 ? 2 : 3), st, nl);
    // SR_SPLIT_KV: the split row-blocks' partial outputs summed into O
    if (e == cudaSuccess && (p.stages & 4) && p.partial) e = launch_combine(p, st, nl);
    return e;
}

cudaError_t launch_tc_unfused(const Params& p, cudaStream_t st, int64_t* nl)
{
    if (p.S > 16384) return cudaErrorNotSupported;  // row buffer of the baseline softmax
    cudaError_t e = cudaSuccess;
    if ((p.stages & 1) && (e = launch_gemm1(p, false, st, nl)) != cudaSuccess) return e;
    if ((p.stages & 2) && (e = launch_softmax(p, st, nl)) != cudaSuccess) return e;
    if (p.stages & 4) e = launch_gemm2(p, 0, st, nl);
    return e;
}

}  // namespace sr
