// Microbenchmark: the I/O skeleton of one TLC row pass at n = 2^22 (2048 x 2048,
// tiles of 4 rows = 8192 words), without the permute arithmetic. Separates the
// cost of the store pattern (64-byte chunks at a 32 KiB stride = the X1 layout)
// from everything else. Persistent grid, one CTA per SM.
//   A ring (TMA 1-D bulk loads of 32 KiB tiles) -> consumer warps copy A -> B
//   (identity, conflict-free) -> B ring -> store mode:
//     0: TMA 1-D bulk store of the whole tile (contiguous, row-major output)
//     1: TMA 3-D tensor store in the X1 geometry (64-byte chunks)
//     2: storer warps, ld.shared.v4 + st.global.v4 in the X1 geometry
//     3: no store (load + copy only)
//     4: consumer warps write the X1 geometry straight from registers (no B ring)
//     5: TMA 2-D tensor store in the X1 geometry with 64-byte box rows
//     6: consumer warps write B, sync among themselves, then st.global.v4 from B
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstring>

namespace {
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile("{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_store_3d(const CUtensorMap* map, const void* src, int c0, int c1, int c2) {
    asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(src)), "r"(c0), "r"(c1), "r"(c2) : "memory");
}
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, const void* src, int c0, int c1) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(src)), "r"(c0), "r"(c1) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N> __device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
}  // namespace

constexpr int HL = 8192;            // words per tile
constexpr int NCONS = 512;          // consumer threads
constexpr int NSTW = 4;             // storer warps (mode 2)

struct Args {
    const uint32_t* in;
    uint32_t* out;
    int ntiles, NA, NB, mode, inflight;
    int r;                           // rows of the view (X1 stride in chunks)
};

extern "C" __global__ void __launch_bounds__(64 + NCONS + 32 * NSTW, 1)
tile_io(const __grid_constant__ CUtensorMap tmap, const __grid_constant__ CUtensorMap tmap2, const Args a) {
    extern __shared__ __align__(128) uint32_t smem[];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int NA = a.NA, NB = a.NB, G = gridDim.x;
    uint32_t* Abuf = smem;
    uint32_t* Bbuf = smem + NA * HL;
    uint64_t* afull = reinterpret_cast<uint64_t*>(Bbuf + NB * HL);
    uint64_t* aempty = afull + NA;
    uint64_t* bfull = aempty + NA;
    uint64_t* bempty = bfull + NB;
    const bool useB = a.mode <= 2 || a.mode == 5;
    if (tid == 0) {
        for (int s = 0; s < NA; ++s) { mbar_init(&afull[s], 1); mbar_init(&aempty[s], NCONS); }
        for (int s = 0; s < NB; ++s) { mbar_init(&bfull[s], NCONS); mbar_init(&bempty[s], a.mode == 2 ? 32 * NSTW : 1); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (warp == 0) {
        if (lane == 0) {
            for (int i = 0;; ++i) {
                const long long t = blockIdx.x + (long long)i * G;
                if (t >= a.ntiles) break;
                const int s = i % NA;
                if (i >= NA) mbar_wait(&aempty[s], (uint32_t)(i / NA - 1) & 1u);
                mbar_arrive_expect_tx(&afull[s], HL * 4u);
                bulk_g2s(Abuf + s * HL, a.in + t * HL, HL * 4u, &afull[s]);
            }
        }
    } else if (warp == 1) {
        if (lane == 0 && (a.mode == 0 || a.mode == 1 || a.mode == 5)) {
            int pending = 0;
            for (int i = 0;; ++i) {
                const long long t = blockIdx.x + (long long)i * G;
                if (t >= a.ntiles) break;
                const int s = i % NB;
                mbar_wait(&bfull[s], (uint32_t)(i / NB) & 1u);
                fence_proxy_async();
                const uint32_t* B = Bbuf + s * HL;
                if (a.mode == 0) bulk_s2g(a.out + t * HL, B, HL * 4u);
                else if (a.mode == 1) { tma_store_3d(&tmap, B, 0, (int)(t * 4), 0); tma_store_3d(&tmap, B + HL / 2, 0, (int)(t * 4), 256); }
                else { tma_store_2d(&tmap2, B, (int)(t * 16), 0); tma_store_2d(&tmap2, B + HL / 2, (int)(t * 16), 256); }
                bulk_commit();
                ++pending;
                // keep at most `inflight` (< NB) stores un-read; free the older B slots in order
                if (pending > a.inflight) {
                    if (a.inflight <= 0) bulk_wait_read<0>(); else if (a.inflight == 1) bulk_wait_read<1>();
                    else if (a.inflight == 2) bulk_wait_read<2>(); else bulk_wait_read<3>();
                    while (pending > a.inflight) {
                        mbar_arrive(&bempty[(i - pending + 1) % NB]);
                        --pending;
                    }
                }
            }
            bulk_wait0();
        }
    } else if (warp < 2 + NCONS / 32) {
        const int ct = tid - 64;
        for (int i = 0;; ++i) {
            const long long t = blockIdx.x + (long long)i * G;
            if (t >= a.ntiles) break;
            const int s = i % NA, sb = i % NB;
            mbar_wait(&afull[s], (uint32_t)(i / NA) & 1u);
            const uint32_t* A = Abuf + s * HL;
            uint32_t v[16];
#pragma unroll
            for (int m = 0; m < 16; ++m) v[m] = A[m * NCONS + ct];
            mbar_arrive(&aempty[s]);
            if (useB) {
                if (i >= NB) mbar_wait(&bempty[sb], (uint32_t)(i / NB - 1) & 1u);
                uint32_t* B = Bbuf + sb * HL;
#pragma unroll
                for (int m = 0; m < 16; ++m) B[m * NCONS + ct] = v[m];
                mbar_arrive(&bfull[sb]);
            } else if (a.mode == 6) {
                uint32_t* B = Bbuf;
                if (i > 0) named_bar(1, NCONS);          // previous tile's B fully read
#pragma unroll
                for (int m = 0; m < 16; ++m) B[m * NCONS + ct] = v[m];
                named_bar(1, NCONS);
                const uint4* B4 = reinterpret_cast<const uint4*>(B);
#pragma unroll
                for (int m = 0; m < 4; ++m) {
                    const int vv = m * NCONS + ct;
                    const long long K = vv >> 2;
                    uint4* dst = reinterpret_cast<uint4*>(a.out + K * a.r * 4 + t * 16) + (vv & 3);
                    *dst = B4[vv];
                }
            } else if (a.mode == 4) {
                // word f = m*NCONS + ct of the tile -> X1 chunk K = f / 16, offset f % 16
#pragma unroll
                for (int m = 0; m < 16; ++m) {
                    const int f = m * NCONS + ct;
                    a.out[(long long)(f >> 4) * a.r * 4 + t * 16 + (f & 15)] = v[m];
                }
            } else {
                uint32_t x = 0;
#pragma unroll
                for (int m = 0; m < 16; ++m) x ^= v[m];
                if (x == 0x12345678u) a.out[0] = x;
            }
        }
    } else if (a.mode == 2) {
        const int st = tid - 64 - NCONS;     // 0 .. 32*NSTW-1
        for (int i = 0;; ++i) {
            const long long t = blockIdx.x + (long long)i * G;
            if (t >= a.ntiles) break;
            const int s = i % NB;
            mbar_wait(&bfull[s], (uint32_t)(i / NB) & 1u);
            const uint4* B4 = reinterpret_cast<const uint4*>(Bbuf + s * HL);
            uint4 v[16];
#pragma unroll
            for (int m = 0; m < 16; ++m) v[m] = B4[m * 32 * NSTW + st];
            mbar_arrive(&bempty[s]);
#pragma unroll
            for (int m = 0; m < 16; ++m) {
                const int vv = m * 32 * NSTW + st;          // 16-byte vector of the tile
                const long long K = vv >> 2;
                uint4* dst = reinterpret_cast<uint4*>(a.out + K * a.r * 4 + t * 16) + (vv & 3);
                *dst = v[m];
            }
        }
    }
}

extern "C" int make_map(CUtensorMap* map, uint32_t* x1, int r, int c) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) return -1;
    auto encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
    const cuuint64_t dims[3] = {4, (cuuint64_t)r, (cuuint64_t)c / 4};
    const cuuint64_t strides[2] = {16, (cuuint64_t)r * 16};
    const cuuint32_t box[3] = {4, 4, 256};
    const cuuint32_t es[3] = {1, 1, 1};
    return encode(map, CU_TENSOR_MAP_DATA_TYPE_UINT32, 3, x1, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS ? 0 : -2;
}

static CUtensorMap g_map, g_map2;
extern "C" int make_map2(CUtensorMap* map, uint32_t* x1, int r, int c) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) return -1;
    auto encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
    const cuuint64_t dims[2] = {(cuuint64_t)r * 4, (cuuint64_t)c / 4};
    const cuuint64_t strides[1] = {(cuuint64_t)r * 16};
    const cuuint32_t box[2] = {16, 256};
    const cuuint32_t es[2] = {1, 1};
    return encode(map, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, x1, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS ? 0 : -2;
}
extern "C" int run(const uint32_t* in, uint32_t* out, int ntiles, int NA, int NB, int mode, int inflight, int grid,
                   cudaStream_t s) {
    static bool init = false;
    static uint32_t* mapped = nullptr;
    if (!init || mapped != out) {
        if (make_map(&g_map, out, 2048, 2048)) return -1;
        if (make_map2(&g_map2, out, 2048, 2048)) return -3;
        init = true; mapped = out;
    }
    Args a{in, out, ntiles, NA, NB, mode, inflight, 2048};
    const size_t smem = (size_t)(NA + NB) * HL * 4 + (2 * NA + 2 * NB) * 8;
    cudaFuncSetAttribute(tile_io, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    tile_io<<<grid, 64 + NCONS + 32 * NSTW, smem, s>>>(g_map, g_map2, a);
    return (int)cudaGetLastError();
}
