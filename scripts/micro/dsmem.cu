// Micro-benchmarks for the cluster designs (DESIGN.md §5 "cluster paths"):
//  mode 0: local smem u32 stores, 32 distinct banks per warp instruction
//  mode 1: DSMEM u32 stores, every lane of a warp to ONE remote CTA (rank+1)
//  mode 2: DSMEM u32 stores, lanes spread over all CTAs of the cluster
//  mode 3: DSMEM u32 loads (16 in flight per thread), one remote CTA per warp
//  mode 4: DSMEM v4 stores, one remote CTA per warp
//  mode 5: cluster barrier (arrive.release + wait.acquire) round trip
// grid_barrier: persistent grid (one CTA per SM), `iters` global-atomic barriers.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t cta_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t n_ctas() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(rank));
    return r;
}
__device__ __forceinline__ void st_cl(uint32_t a, uint32_t v) {
    asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void st_cl4(uint32_t a, uint4 v) {
    asm volatile("st.shared::cluster.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}
__device__ __forceinline__ uint32_t ld_cl(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}

extern "C" __global__ void __launch_bounds__(1024, 1) dsmem_kernel(int mode, int iters, unsigned long long* out) {
    extern __shared__ __align__(128) uint32_t sm[];
    constexpr int WORDS = 16384;   // 64 KiB
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t me = cta_rank(), C = n_ctas();
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
    for (int i = tid; i < WORDS; i += blockDim.x) sm[i] = i;
    cluster_sync();
    const unsigned long long t0 = clock64();
    uint32_t acc = 0;
    if (mode == 5) {
        for (int it = 0; it < iters; ++it) cluster_sync();
    } else {
        for (int it = 0; it < iters; ++it) {
            // 16 words per thread per iteration: warp w, step m -> words (w*16 + m)*32 + lane
#pragma unroll
            for (int m = 0; m < 16; ++m) {
                const uint32_t word = ((warp * 16 + m) * 32 + lane) & (WORDS - 1);
                const uint32_t la = base + word * 4;
                if (mode == 0) {
                    asm volatile("st.shared.u32 [%0], %1;" ::"r"(la), "r"(word + it) : "memory");
                } else if (mode == 1) {
                    st_cl(mapa(la, (me + 1) % C), word + it);
                } else if (mode == 2) {
                    st_cl(mapa(la, (me + 1 + lane) % C), word + it);
                } else if (mode == 3) {
                    acc += ld_cl(mapa(la, (me + 1) % C));
                } else if (mode == 4) {
                    if (m < 4) {
                        const uint32_t w4 = ((warp * 4 + m) * 32 + lane) * 4 & (WORDS - 1);
                        st_cl4(mapa(base + w4 * 4, (me + 1) % C), make_uint4(w4, it, 1, 2));
                    }
                }
            }
        }
    }
    cluster_sync();
    const unsigned long long t1 = clock64();
    if (tid == 0) out[blockIdx.x] = t1 - t0;
    if (acc == 0xdeadbeef) out[0] = 0;
}

extern "C" __global__ void grid_barrier_kernel(int iters, unsigned long long* ctr, unsigned long long* out) {
    const unsigned long long t0 = clock64();
    const unsigned long long G = gridDim.x;
    for (int it = 1; it <= iters; ++it) {
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            asm volatile("red.release.gpu.global.add.u64 [%0], 1;" ::"l"(ctr) : "memory");
            unsigned long long v;
            do {
                asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(ctr) : "memory");
            } while (v < G * it);
        }
        __syncthreads();
    }
    const unsigned long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}

extern "C" int run_dsmem(int mode, int csize, int grid, int iters, unsigned long long* out, float* ms) {
    cudaFuncSetAttribute(dsmem_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
    cudaFuncSetAttribute(dsmem_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(1024);
    cfg.dynamicSmemBytes = 65536;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = csize;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    cudaError_t e = cudaLaunchKernelEx(&cfg, dsmem_kernel, mode, iters, out);
    cudaEventRecord(e1);
    if (e != cudaSuccess) { printf("launch: %s\n", cudaGetErrorString(e)); return -1; }
    e = cudaEventSynchronize(e1);
    if (e != cudaSuccess) { printf("sync: %s\n", cudaGetErrorString(e)); return -2; }
    cudaEventElapsedTime(ms, e0, e1);
    return 0;
}

extern "C" int run_grid_barrier(int grid, int threads, int iters, unsigned long long* ctr, unsigned long long* out, float* ms) {
    cudaMemset(ctr, 0, 8);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    grid_barrier_kernel<<<grid, threads>>>(iters, ctr, out);
    cudaEventRecord(e1);
    cudaError_t e = cudaEventSynchronize(e1);
    if (e != cudaSuccess) { printf("sync: %s\n", cudaGetErrorString(e)); return -2; }
    cudaEventElapsedTime(ms, e0, e1);
    return 0;
}
