#include <cstdio>
#include <cstdint>
struct Blob { int32_t n; int32_t w[6000]; };
struct Ptrs { const int32_t* a; };
__device__ __forceinline__ int32_t sld(const int32_t* p) { return *p; }
__global__ void k(const __grid_constant__ Blob b, int32_t* out, const int32_t* g)
{
    __shared__ Ptrs sh;
    if (threadIdx.x == 0) sh.a = (b.n > 0) ? &b.w[0] : g;
    __syncthreads();
    int32_t s = 0;
    for (int i = threadIdx.x; i < 6000; i += blockDim.x) s += sld(sh.a + i);
    atomicAdd(out, s);
}
int main() {
    static Blob b; b.n = 6000; long want = 0;
    for (int i = 0; i < 6000; ++i) { b.w[i] = i * 7 + 1; want += b.w[i]; }
    int32_t* o; int32_t* g; cudaMalloc(&o, 4); cudaMalloc(&g, 6000 * 4); cudaMemset(o, 0, 4);
    cudaMemcpy(g, b.w, 6000 * 4, cudaMemcpyHostToDevice);
    k<<<4, 256>>>(b, o, g);
    int32_t h; cudaMemcpy(&h, o, 4, cudaMemcpyDeviceToHost);
    printf("param-space generic loads: %d (expect %ld) err=%s\n", h, 4 * want, cudaGetErrorString(cudaGetLastError()));
    b.n = 0; cudaMemset(o, 0, 4); k<<<4, 256>>>(b, o, g); cudaMemcpy(&h, o, 4, cudaMemcpyDeviceToHost);
    printf("global via same path: %d (expect %ld)\n", h, 4 * want);
}
