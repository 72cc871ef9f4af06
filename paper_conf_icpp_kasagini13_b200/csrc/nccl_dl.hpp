// nccl_dl.hpp — the few NCCL entry points the row-sharded apply uses,
// resolved at run time with dlopen so libperm links without NCCL and picks up the
// NCCL already loaded in the process (PyTorch's, when torch.distributed is in use).
// Only the column phase's two all-to-all exchanges (Lemma 8) go
// through NCCL; everything else is libperm's kernels.
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>

#include <cstdint>
#include <string>

namespace perm {

struct NcclApi {
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
    ncclResult_t (*GetVersion)(int*) = nullptr;
};

// The process-wide table, loaded on first use; nullptr (with `err` set) when no
// libnccl.so.2 can be opened or a symbol is missing.
const NcclApi* nccl_api(std::string& err);

// All-to-all of `world` uniform blocks of `block_words` 32-bit words on `comm`:
// recv[q*B : (q+1)*B] <- peer q's send[rank*B : (rank+1)*B], stream-ordered
// (grouped point-to-point send/recv, one pair per peer).
ncclResult_t nccl_alltoall(const NcclApi& api, const uint32_t* send, uint32_t* recv, int64_t block_words,
                           int world, ncclComm_t comm, cudaStream_t s);

}  // namespace perm
