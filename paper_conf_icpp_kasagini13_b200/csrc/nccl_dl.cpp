// nccl_dl.cpp — run-time binding of NCCL for the row-sharded apply (see nccl_dl.hpp).
#include "nccl_dl.hpp"

#include <dlfcn.h>

#include <mutex>

namespace perm {

namespace {

template <class F>
bool load(void* h, const char* name, F& fn) {
    fn = reinterpret_cast<F>(dlsym(h, name));
    return fn != nullptr;
}

}  // namespace

const NcclApi* nccl_api(std::string& err) {
    static NcclApi api;
    static std::string load_err;
    static bool ok = false;
    static std::once_flag once;
    std::call_once(once, [] {
        // an NCCL already mapped into the process first (torch's), then the loader's search
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            const char* e = dlerror();
            load_err = std::string("cannot open libnccl.so.2: ") + (e ? e : "?");
            return;
        }
        ok = load(h, "ncclGetUniqueId", api.GetUniqueId) && load(h, "ncclCommInitRank", api.CommInitRank) &&
             load(h, "ncclCommDestroy", api.CommDestroy) && load(h, "ncclSend", api.Send) &&
             load(h, "ncclRecv", api.Recv) && load(h, "ncclGroupStart", api.GroupStart) &&
             load(h, "ncclGroupEnd", api.GroupEnd) && load(h, "ncclGetErrorString", api.GetErrorString) &&
             load(h, "ncclGetVersion", api.GetVersion);
        if (!ok) load_err = "libnccl.so.2 lacks a required symbol";
    });
    if (!ok) {
        err = load_err;
        return nullptr;
    }
    return &api;
}

ncclResult_t nccl_alltoall(const NcclApi& api, const uint32_t* send, uint32_t* recv, int64_t block_words,
                           int world, ncclComm_t comm, cudaStream_t s) {
    ncclResult_t r = api.GroupStart();
    for (int q = 0; q < world && r == ncclSuccess; ++q) {
        r = api.Send(send + (int64_t)q * block_words, (size_t)block_words, ncclUint32, q, comm, s);
        if (r == ncclSuccess)
            r = api.Recv(recv + (int64_t)q * block_words, (size_t)block_words, ncclUint32, q, comm, s);
    }
    const ncclResult_t e = api.GroupEnd();
    return r != ncclSuccess ? r : e;
}

}  // namespace perm
