// Microbenchmark: global store throughput of the LINES-layout column-chunk pattern.
// Each CTA writes tiles of h lines x L positions: element (l, pos) of tile t goes
// to out[pos * R + t * h + l] (column-major), as 128-bit vectors of 4 consecutive l.
#include <cuda_runtime.h>
#include <cstdint>
extern "C" __global__ void cross_store(uint32_t* out, int L, int R, int h, int ntiles, int coalesced) {
    const int T = blockDim.x;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int nv = h * L / 4;
        for (int v = threadIdx.x; v < nv; v += T) {
            const int f = 4 * v;
            uint4 val = make_uint4(f, f + 1, f + 2, f + 3);
            long long idx;
            if (coalesced) idx = (long long)t * h * L + f;
            else {
                const int pos = f / h, l = f % h;
                idx = (long long)pos * R + (long long)t * h + l;
            }
            *reinterpret_cast<uint4*>(out + idx) = val;
        }
    }
}
extern "C" int run(uint32_t* out, int L, int R, int h, int ntiles, int coalesced, int grid, int block) {
    cross_store<<<grid, block>>>(out, L, R, h, ntiles, coalesced);
    return (int)cudaGetLastError();
}
