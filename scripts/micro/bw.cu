// In-kernel (globaltimer) bandwidth of coalesced writes / reads / copies, to separate
// kernel time from launch latency.
#include <cuda_runtime.h>
#include <cstdint>
__device__ __forceinline__ unsigned long long gt() { unsigned long long t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }
extern "C" __global__ void k_write(uint4* out, long long nv, unsigned long long* ts) {
    if (threadIdx.x == 0) ts[2 * blockIdx.x] = gt();
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nv; v += (long long)gridDim.x * blockDim.x)
        out[v] = make_uint4(v, v, v, v);
    __syncthreads();
    if (threadIdx.x == 0) ts[2 * blockIdx.x + 1] = gt();
}
extern "C" __global__ void k_copy(const uint4* in, uint4* out, long long nv, unsigned long long* ts) {
    if (threadIdx.x == 0) ts[2 * blockIdx.x] = gt();
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nv; v += (long long)gridDim.x * blockDim.x)
        out[v] = in[v];
    __syncthreads();
    if (threadIdx.x == 0) ts[2 * blockIdx.x + 1] = gt();
}
extern "C" __global__ void k_read(const uint4* in, long long nv, unsigned long long* ts, unsigned* sink) {
    if (threadIdx.x == 0) ts[2 * blockIdx.x] = gt();
    unsigned acc = 0;
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < nv; v += (long long)gridDim.x * blockDim.x) {
        uint4 x = in[v]; acc ^= x.x ^ x.y ^ x.z ^ x.w;
    }
    if (acc == 0x12345678) *sink = acc;
    __syncthreads();
    if (threadIdx.x == 0) ts[2 * blockIdx.x + 1] = gt();
}
extern "C" int run(int kind, void* in, void* out, long long nv, unsigned long long* ts, unsigned* sink, int grid, int block) {
    if (kind == 0) k_write<<<grid, block>>>((uint4*)out, nv, ts);
    else if (kind == 1) k_copy<<<grid, block>>>((const uint4*)in, (uint4*)out, nv, ts);
    else k_read<<<grid, block>>>((const uint4*)in, nv, ts, sink);
    return (int)cudaGetLastError();
}
