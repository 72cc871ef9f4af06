// capi.cpp — the C ABI of libperm (include/perm.h): plan lifecycle, error
// model, device memory and the launch sequence of perm_apply.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>

#include "../../include/perm.h"
#include "kernels.hpp"
#include "nccl_dl.hpp"
#include "plan.hpp"

using perm::HostPlan;

struct perm_plan {
    HostPlan host;
    bool on_device = false;
    int device = -1;
    uint32_t* d_sched = nullptr;          // the three phases back to back
    uint32_t* d_phase[3] = {nullptr, nullptr, nullptr};
    uint32_t* d_scratch[2] = {nullptr, nullptr};
    int64_t sched_bytes = 0, scratch_bytes = 0;
    double ms_upload = 0;
    // staging for perm_apply_host
    uint32_t* d_stage[2] = {nullptr, nullptr};
    // profiling
    bool profiling = false;
    int n_events = 0;
    cudaEvent_t ev[8] = {};
    int last_kernels = 0;
    // tracing: [row pass][cta][16] %globaltimer stamps
    unsigned long long* d_trace = nullptr;
    int64_t trace_stride = 0;          // CTAs per pass slot
    unsigned long long* d_sync = nullptr;   // fused 3-pass grid-barrier counters
    int32_t* d_p = nullptr;                 // low-distribution shortcut: q = P^-1 (or p)
    alignas(64) CUtensorMap tlc_maps[3];   // TLC layout: TMA tensor maps of X1, X2
    // row-sharded plans created with an NCCL unique id: the communicator of the
    // column phase's two all-to-alls and the plan-owned send / receive shards
    ncclComm_t comm = nullptr;
    uint32_t* d_send = nullptr;
    uint32_t* d_recv = nullptr;
};

namespace {

thread_local int g_status = PERM_OK;
thread_local std::string g_msg = "ok";

int fail(int status, const std::string& msg) {
    g_status = status;
    g_msg = msg;
    return status;
}

int cuda_fail(cudaError_t e, const char* what) {
    return fail(PERM_ECUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

void free_device(perm_plan* pl) {
    if (!pl->on_device) return;
    int cur = -1;
    cudaGetDevice(&cur);
    if (pl->device >= 0) cudaSetDevice(pl->device);
    cudaFree(pl->d_sched);
    cudaFree(pl->d_scratch[0]);
    cudaFree(pl->d_scratch[1]);
    cudaFree(pl->d_stage[0]);
    cudaFree(pl->d_stage[1]);
    cudaFree(pl->d_trace);
    cudaFree(pl->d_sync);
    cudaFree(pl->d_p);
    cudaFree(pl->d_send);
    cudaFree(pl->d_recv);
    if (pl->comm) {
        std::string err;
        if (const perm::NcclApi* api = perm::nccl_api(err)) api->CommDestroy(pl->comm);
        pl->comm = nullptr;
    }
    for (int i = 0; i < pl->n_events; ++i) cudaEventDestroy(pl->ev[i]);
    pl->n_events = 0;
    if (cur >= 0) cudaSetDevice(cur);
    pl->on_device = false;
}

int upload(perm_plan* pl) {
    auto t0 = std::chrono::steady_clock::now();
    HostPlan& P = pl->host;
    cudaError_t e = cudaGetDevice(&pl->device);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice");
    auto padded = [](int64_t w) { return (w + 32 + 63) / 64 * 64; };   // guard, 256-B aligned phases
    int64_t words = 0;
    for (int f = 0; f < 3; ++f) words += padded((int64_t)P.sched[f].size());
    pl->sched_bytes = words * 4;
    e = cudaMalloc(&pl->d_sched, (size_t)pl->sched_bytes);
    if (e != cudaSuccess) return fail(PERM_ENOMEM, std::string("cudaMalloc schedules: ") + cudaGetErrorString(e));
    pl->on_device = true;
    int64_t off = 0;
    for (int f = 0; f < 3; ++f) {
        pl->d_phase[f] = pl->d_sched + off;
        const int64_t wf = (int64_t)P.sched[f].size();
        e = cudaMemcpy(pl->d_phase[f], P.sched[f].data(), (size_t)wf * 4, cudaMemcpyHostToDevice);
        if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpy schedules");
        e = cudaMemset(pl->d_phase[f] + wf, 0, 32 * 4);
        if (e != cudaSuccess) return cuda_fail(e, "cudaMemset");
        off += padded(wf);
    }
    if (P.passes > 2) {
        const size_t bytes = (size_t)(P.r_l ? P.n / P.world : P.n) * P.eb;
        for (int i = 0; i < 2; ++i) {
            e = cudaMalloc(&pl->d_scratch[i], bytes);
            if (e != cudaSuccess) return fail(PERM_ENOMEM, std::string("cudaMalloc scratch: ") + cudaGetErrorString(e));
        }
        pl->scratch_bytes = 2 * (int64_t)bytes;
    }
    e = perm::prepare_kernels(P);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute");
    if (P.direct) {
        e = cudaMalloc(&pl->d_p, P.p_copy.size() * sizeof(int32_t));
        if (e == cudaSuccess)
            e = cudaMemcpy(pl->d_p, P.p_copy.data(), P.p_copy.size() * sizeof(int32_t), cudaMemcpyHostToDevice);
        if (e != cudaSuccess) return cuda_fail(e, "upload p (direct)");
        std::vector<int32_t>().swap(pl->host.p_copy);
    }
    if (P.layout == 3 || P.layout == 5) {
        e = perm::make_tlc_maps(P, pl->d_scratch[0], pl->d_scratch[1], pl->tlc_maps);
        if (e != cudaSuccess) return cuda_fail(e, "cuTensorMapEncodeTiled");
    }
    if (P.fused3) {
        e = cudaMalloc(&pl->d_sync, 4 * sizeof(unsigned long long));
        if (e == cudaSuccess) e = cudaMemset(pl->d_sync, 0, 4 * sizeof(unsigned long long));
        if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc sync");
    }
    for (int i = 0; i < 8; ++i) {
        e = cudaEventCreate(&pl->ev[i]);
        if (e != cudaSuccess) return cuda_fail(e, "cudaEventCreate");
        pl->n_events = i + 1;
    }
    e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceSynchronize");
    pl->ms_upload =
        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return PERM_OK;
}

perm_plan* create(const int32_t* p, int64_t n, int32_t eb, const perm_plan_options* opt,
                  bool device, int world = 0, int rank = 0) {
    perm_plan* pl = new (std::nothrow) perm_plan();
    if (!pl) { fail(PERM_ENOMEM, "out of host memory"); return nullptr; }
    std::string err;
    int st;
    // where the colourings run: auto -> the device for device plans with n >= 2^20
    perm_plan_options o{};
    if (opt) o = *opt;
    if (o.gpu_planner == 0) o.gpu_planner = (device && n >= (int64_t(1) << 20)) ? 1 : -1;
    try {
        st = world > 0 ? perm::build_sharded_plan(p, n, eb, world, rank, &o, pl->host, err)
                       : perm::build_host_plan(p, n, eb, &o, pl->host, err);
    } catch (const std::bad_alloc&) {
        st = PERM_ENOMEM;
        err = "out of host memory while planning";
    }
    if (st != PERM_OK) {
        fail(st, err);
        delete pl;
        return nullptr;
    }
    if (device) {
        st = upload(pl);
        if (st != PERM_OK) {
            free_device(pl);
            delete pl;
            return nullptr;
        }
    }
    g_status = PERM_OK;
    g_msg = "ok";
    return pl;
}

int nccl_fail(const perm::NcclApi* api, ncclResult_t r, const char* what) {
    return fail(PERM_ENCCL, std::string(what) + ": " + (api ? api->GetErrorString(r) : "NCCL unavailable"));
}

// NCCL communicator + exchange buffers of a sharded device plan (collective over the ranks)
int attach_comm(perm_plan* pl, const void* uid) {
    std::string err;
    const perm::NcclApi* api = perm::nccl_api(err);
    if (!api) return fail(PERM_ENCCL, err);
    const HostPlan& P = pl->host;
    ncclUniqueId id;
    std::memcpy(&id, uid, sizeof(id));
    cudaError_t e = cudaSetDevice(pl->device);
    if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
    const ncclResult_t r = api->CommInitRank(&pl->comm, P.world, id, P.rank);
    if (r != ncclSuccess) {
        pl->comm = nullptr;
        return nccl_fail(api, r, "ncclCommInitRank");
    }
    const size_t bytes = (size_t)(P.n / P.world) * P.eb;
    e = cudaMalloc(&pl->d_send, bytes);
    if (e == cudaSuccess) e = cudaMalloc(&pl->d_recv, bytes);
    if (e != cudaSuccess) return fail(PERM_ENOMEM, std::string("cudaMalloc exchange buffers: ") + cudaGetErrorString(e));
    return PERM_OK;
}

bool overlap(const void* a, const void* b, int64_t bytes) {
    const char* x = static_cast<const char*>(a);
    const char* y = static_cast<const char*>(b);
    return x < y + bytes && y < x + bytes;
}

}  // namespace

extern "C" {

perm_plan* perm_plan_create(const int32_t* p, int64_t n, int32_t elem_bytes) {
    return create(p, n, elem_bytes, nullptr, true);
}

perm_plan* perm_plan_create_ex(const int32_t* p, int64_t n, int32_t elem_bytes,
                               const perm_plan_options* opt) {
    return create(p, n, elem_bytes, opt, true);
}

perm_plan* perm_plan_create_host(const int32_t* p, int64_t n, int32_t elem_bytes,
                                 const perm_plan_options* opt) {
    return create(p, n, elem_bytes, opt, false);
}

int perm_nccl_unique_id(void* uid_out) {
    if (!uid_out) return fail(PERM_EINVAL, "null uid buffer");
    std::string err;
    const perm::NcclApi* api = perm::nccl_api(err);
    if (!api) return fail(PERM_ENCCL, err);
    ncclUniqueId id;
    const ncclResult_t r = api->GetUniqueId(&id);
    if (r != ncclSuccess) return nccl_fail(api, r, "ncclGetUniqueId");
    std::memcpy(uid_out, &id, sizeof(id));
    return PERM_OK;
}

perm_plan* perm_plan_create_sharded_ex(const int32_t* p, int64_t n, int32_t elem_bytes, int32_t world,
                                       int32_t rank, const void* nccl_uid, const perm_plan_options* opt) {
    if (world < 1) { fail(PERM_EINVAL, "world must be >= 1"); return nullptr; }
    perm_plan* pl = create(p, n, elem_bytes, opt, true, world, rank);
    if (!pl || !nccl_uid) return pl;
    if (attach_comm(pl, nccl_uid) != PERM_OK) {
        const int st = g_status;
        const std::string msg = g_msg;
        free_device(pl);
        delete pl;
        fail(st, msg);
        return nullptr;
    }
    return pl;
}

perm_plan* perm_plan_create_sharded(const int32_t* p, int64_t n, int32_t elem_bytes, int32_t world,
                                    int32_t rank, const void* nccl_uid) {
    return perm_plan_create_sharded_ex(p, n, elem_bytes, world, rank, nccl_uid, nullptr);
}

int perm_sharded_exchange(const perm_plan* plan, const void* send, void* recv, perm_stream_t stream) {
    if (!plan || !send || !recv) return fail(PERM_EINVAL, "null plan or buffer");
    const HostPlan& P = plan->host;
    if (!P.r_l) return fail(PERM_EINVAL, "not a row-sharded plan");
    if (!plan->comm) return fail(PERM_ENCCL, "plan has no NCCL communicator (created without nccl_uid)");
    if (overlap(send, recv, P.n / P.world * P.eb)) return fail(PERM_EINVAL, "send and recv overlap");
    std::string err;
    const perm::NcclApi* api = perm::nccl_api(err);
    if (!api) return fail(PERM_ENCCL, err);
    const int64_t block = P.n / ((int64_t)P.world * P.world);
    const ncclResult_t r = perm::nccl_alltoall(*api, static_cast<const uint32_t*>(send), static_cast<uint32_t*>(recv),
                                               block, P.world, plan->comm, static_cast<cudaStream_t>(stream));
    if (r != ncclSuccess) return nccl_fail(api, r, "all-to-all");
    return PERM_OK;
}

int perm_apply_sharded(const perm_plan* plan, const void* a_shard, void* b_shard, perm_stream_t stream) {
    if (!plan || !a_shard || !b_shard) return fail(PERM_EINVAL, "null plan or buffer");
    if (!plan->on_device) return fail(PERM_ENODEVICE, "plan was created host-only");
    const HostPlan& P = plan->host;
    if (!P.r_l) return fail(PERM_EINVAL, "not a row-sharded plan (use perm_apply)");
    if (!plan->comm) return fail(PERM_ENCCL, "plan has no NCCL communicator (created without nccl_uid)");
    if (overlap(a_shard, b_shard, P.n / P.world * P.eb)) return fail(PERM_EINVAL, "a and b shards overlap");
    // step 0 -> all-to-all -> step 1 -> all-to-all -> step 2 (Lemma 8: the column phase's two
    // transposes become the two uniform, P-independent exchanges; in the TLC form the steps
    // write / read the exchange layouts directly, in the per-line form steps 0 and 1 add a
    // transpose)
    int st = perm_sharded_step(plan, 0, a_shard, plan->d_send, stream);
    if (st == PERM_OK) st = perm_sharded_exchange(plan, plan->d_send, plan->d_recv, stream);
    if (st == PERM_OK) st = perm_sharded_step(plan, 1, plan->d_recv, plan->d_send, stream);
    if (st == PERM_OK) st = perm_sharded_exchange(plan, plan->d_send, plan->d_recv, stream);
    if (st == PERM_OK) st = perm_sharded_step(plan, 2, plan->d_recv, b_shard, stream);
    return st;
}

perm_plan* perm_plan_create_sharded_host(const int32_t* p, int64_t n, int32_t elem_bytes,
                                         int32_t world, int32_t rank, const perm_plan_options* opt) {
    return create(p, n, elem_bytes, opt, false, world, rank);
}

int perm_sharded_step(const perm_plan* plan, int32_t step, const void* in, void* out,
                      perm_stream_t stream) {
    if (!plan || !in || !out) return fail(PERM_EINVAL, "null plan or buffer");
    if (!plan->on_device) return fail(PERM_ENODEVICE, "plan was created host-only");
    const HostPlan& P = plan->host;
    if (!P.r_l) return fail(PERM_EINVAL, "not a row-sharded plan");
    const int64_t shard = P.n / P.world;
    if (overlap(in, out, shard * P.eb)) return fail(PERM_EINVAL, "in and out overlap");
    if ((reinterpret_cast<uintptr_t>(in) | reinterpret_cast<uintptr_t>(out)) & 15)
        return fail(PERM_EINVAL, "buffers must be 16-byte aligned");
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const uint32_t* src = static_cast<const uint32_t*>(in);
    uint32_t* dst = static_cast<uint32_t*>(out);
    cudaError_t e;
    if (P.layout == 3) {
        // TLC form: one tile-coloured pass per step, writing the exchange layout directly
        // (step 0: X1 of my rows = per-peer column blocks; step 1: X2 of my columns = per-peer
        // row blocks; step 2: rows of b) and reading received tiles as one segment per sender
        if (step < 0 || step > 2) return fail(PERM_EINVAL, "step must be 0, 1 or 2");
        alignas(64) CUtensorMap maps[3] = {};
        if (step < 2) {
            e = perm::make_tlc_maps(P, dst, dst, maps);
            if (e != cudaSuccess) return cuda_fail(e, "cuTensorMapEncodeTiled (sharded)");
        }
        e = perm::launch_tlc_pass(P, step, maps, plan->d_phase[step], src, dst, s, false, nullptr);
        if (e != cudaSuccess) return cuda_fail(e, "sharded step launch");
        return PERM_OK;
    }
    if (step == 0) {          // R1 on my rows, then T-pack: (r_l x c) -> (c x r_l), peer q = rows q*c_l..
        e = perm::launch_row_pass(P, 0, plan->d_phase[0], src, plan->d_scratch[0], s, false);
        if (e == cudaSuccess) e = perm::launch_transpose(plan->d_scratch[0], dst, P.r_l, P.c, s, true);
    } else if (step == 1) {   // R2 on my columns (segments from every sender), T-pack: (c_l x r) -> (r x c_l)
        e = perm::launch_row_pass(P, 1, plan->d_phase[1], src, plan->d_scratch[1], s, false);
        if (e == cudaSuccess) e = perm::launch_transpose(plan->d_scratch[1], dst, P.c_l, P.r, s, true);
    } else if (step == 2) {   // R3 on my rows (segments from every sender) -> b shard
        e = perm::launch_row_pass(P, 2, plan->d_phase[2], src, dst, s, false);
    } else {
        return fail(PERM_EINVAL, "step must be 0, 1 or 2");
    }
    if (e != cudaSuccess) return cuda_fail(e, "sharded step launch");
    return PERM_OK;
}

void perm_plan_destroy(perm_plan* plan) {
    if (!plan) return;
    free_device(plan);
    delete plan;
}

int perm_plan_get_info(const perm_plan* plan, perm_plan_info* out) {
    if (!plan || !out) return fail(PERM_EINVAL, "null plan or info");
    const HostPlan& P = plan->host;
    std::memset(out, 0, sizeof(*out));
    out->n = P.user_n;
    out->rows = P.r;
    out->cols = P.c;
    int64_t words = 0;
    for (int f = 0; f < 3; ++f) words += (int64_t)P.sched[f].size();
    out->sched_bytes = plan->on_device ? plan->sched_bytes : words * 4;
    out->scratch_bytes = plan->on_device ? plan->scratch_bytes : (P.passes > 2 ? 2 * P.n * P.eb : 0);
    out->elem_bytes = P.user_eb;
    out->passes = P.passes;
    out->kernels_per_apply = (plan->d_p || P.fused3 || P.passes == 2) ? 1 : P.passes;
    out->distribution = P.distribution;
    out->direct = P.direct;
    out->gpu_planner = P.gpu_planner;
    for (int f = 0; f < 3; ++f) {
        out->entry_bits[f] = P.layout >= 3 ? P.tp[f].E : P.ph[f].E;
        out->h[f] = P.passes == 1 ? (int32_t)P.ph[f].lines : (P.layout == 5 ? P.tp[f].h : P.rp[f].h);
    }
    out->planner_threads = P.threads_used;
    out->build_ms_colour = P.ms_colour;
    out->build_ms_bank = P.ms_bank;
    out->build_ms_upload = plan->ms_upload;
    out->world = P.r_l ? P.world : 1;
    out->rank = P.r_l ? P.rank : 0;
    const int64_t wpe = P.user_eb / 4;          // words per caller element
    out->shard_elems = (P.r_l ? P.n / P.world : P.n) / wpe;
    out->block_elems = (P.r_l ? P.n / ((int64_t)P.world * P.world) : P.n) / wpe;
    return PERM_OK;
}

int64_t perm_plan_describe(const perm_plan* plan, char* buf, int64_t len) {
    if (!plan) return fail(PERM_EINVAL, "null plan");
    const HostPlan& P = plan->host;
    std::string s = "{\"n\":" + std::to_string(P.n) + ",\"rows\":" + std::to_string(P.r) +
                    ",\"cols\":" + std::to_string(P.c) + ",\"passes\":" + std::to_string(P.passes) +
                    ",\"layout\":" + std::to_string(P.layout) + ",\"fused3\":" + std::to_string(P.fused3) +
                    ",\"distribution\":" + std::to_string(P.distribution) +
                    ",\"direct\":" + std::to_string(P.direct);
    if (P.passes == 2) s += ",\"cluster\":" + std::to_string(P.cluster);
    if (P.layout >= 3) {
        s += ",\"tlc\":[";
        for (int f = 0; f < 3; ++f) {
            const perm::TlcPass& tp = P.tp[f];
            s += std::string(f ? "," : "") + "{\"h\":" + std::to_string(tp.h) + ",\"HL\":" +
                 std::to_string(tp.HL) + ",\"E\":" + std::to_string(tp.E) + ",\"ept\":" +
                 std::to_string(tp.ept) + ",\"nwords\":" + std::to_string(tp.nwords) +
                 ",\"ntiles\":" + std::to_string(tp.ntiles) + ",\"stages\":" +
                 std::to_string(tp.stages) + ",\"grid\":" + std::to_string(tp.grid) +
                 ",\"out_kind\":" + std::to_string(tp.out_kind) + "}";
        }
        s += "]";
    }
    if (P.passes == 1) {
        s += ",\"fused\":{\"threads\":" + std::to_string(P.fused_threads) + ",\"ept\":" +
             std::to_string(P.fused_ept) + ",\"Ls\":" + std::to_string(P.fused_Ls) + "}";
    } else {
        s += ",\"row_passes\":[";
        for (int f = 0; f < 3; ++f) {
            const perm::RowPass& rp = P.rp[f];
            auto io = [](const perm::IoMode& m) {
                return std::string("{\"cross\":") + std::to_string(m.cross) + ",\"w\":" +
                       std::to_string(m.w) + ",\"strideK\":" + std::to_string(m.strideK) +
                       ",\"blockP\":" + std::to_string(m.blockP) + ",\"strideP\":" +
                       std::to_string(m.strideP) + ",\"cta_stride\":" + std::to_string(m.cta_stride) + "}";
            };
            s += std::string(f ? "," : "") + "{\"phase\":" + std::to_string(rp.phase) +
                 ",\"tma\":" + std::to_string(rp.tma) + ",\"sg\":" + std::to_string(rp.sg) + ",\"split\":" + std::to_string(rp.split) + ",\"stages\":" + std::to_string(rp.stages) +
                 ",\"grid\":" + std::to_string(rp.grid) +
                 ",\"L\":" + std::to_string(P.ph[rp.phase].L) + ",\"E\":" +
                 std::to_string(P.ph[rp.phase].E) + ",\"dense\":" + std::to_string(P.ph[rp.phase].dense) +
                 ",\"sched_words_per_line\":" + std::to_string(P.ph[rp.phase].wpl) +
                 ",\"h\":" + std::to_string(rp.h) +
                 ",\"ctas\":" + std::to_string(rp.ctas) + ",\"threads\":" +
                 std::to_string(rp.threads) + ",\"ept\":" + std::to_string(rp.ept) +
                 ",\"Ls\":" + std::to_string(rp.Ls) + ",\"smem_bytes\":" +
                 std::to_string((int64_t)rp.h * rp.Ls * 4) + ",\"wavefronts_in\":" +
                 std::to_string(rp.conflicts_in) + ",\"wavefronts_out\":" +
                 std::to_string(rp.conflicts_out) + ",\"in\":" + io(rp.in) + ",\"out\":" +
                 io(rp.out) + "}";
        }
        s += "]";
    }
    s += "}";
    if (buf && len > 0) {
        const int64_t m = std::min<int64_t>(len - 1, (int64_t)s.size());
        std::memcpy(buf, s.data(), (size_t)m);
        buf[m] = 0;
    }
    return (int64_t)s.size() + 1;
}

int perm_plan_export(const perm_plan* plan, uint16_t* kappa, uint32_t* s1, uint32_t* s2,
                     uint32_t* s3) {
    if (!plan) return fail(PERM_EINVAL, "null plan");
    const HostPlan& P = plan->host;
    if (P.direct) return fail(PERM_EUNSUPPORTED, "low-distribution shortcut plan: no schedule to export");
    if (kappa) std::memcpy(kappa, P.kappa.data(), (size_t)P.n * sizeof(uint16_t));   // words
    uint32_t* outs[3] = {s1, s2, s3};
    if (P.layout == 5) {
        // TLC ring: tile T's entries in the dense per-round format of a 32768-word line
        for (int f = 0; f < 3; ++f) {
            if (!outs[f]) continue;
            const perm::PhaseGeom& g = P.ph[f];
#pragma omp parallel for schedule(static)
            for (int64_t T = 0; T < g.lines; ++T)
                for (int64_t q = 0; q < g.L; ++q) {
                    const uint32_t e = perm::unpack_entry(P.sched[f], g, T, q);
                    const uint32_t src = ((e >> g.logL) << 5) | (uint32_t)(q & 31);
                    const uint32_t dst = e & ((1u << g.logL) - 1u);
                    outs[f][T * g.L + q] = (src << 16) | dst;
                }
        }
        return PERM_OK;
    }
    if (P.layout >= 3) {
        // TLC / cluster path: entry (tile T, round q, lane x) -> (src word offset in A << 16) | dst offset in B
        for (int f = 0; f < 3; ++f) {
            if (!outs[f]) continue;
            const perm::TlcPass& tp = P.tp[f];
#pragma omp parallel for schedule(static)
            for (int64_t T = 0; T < tp.ntiles; ++T)
                for (int64_t q = 0; q < tp.HL / 32; ++q)
                    for (int64_t x = 0; x < 32; ++x) {
                        const uint32_t e = perm::tlc_entry(P.sched[f], tp, T, q, x);
                        const uint32_t src = ((e >> tp.dec.lt) << 5) | (uint32_t)x;
                        const uint32_t dst = perm::tlc_dst(tp.dec, e & ((1u << tp.dec.lt) - 1u), src);
                        outs[f][T * tp.HL + q * 32 + x] = (src << 16) | dst;
                    }
        }
        return PERM_OK;
    }
    for (int f = 0; f < 3; ++f) {
        if (!outs[f]) continue;
        const perm::PhaseGeom& g = P.ph[f];
        const uint32_t tmask = (1u << g.logL) - 1u;
#pragma omp parallel for schedule(static)
        for (int64_t line = 0; line < g.lines; ++line) {
            for (int64_t q = 0; q < g.L; ++q) {
                const uint32_t e = perm::unpack_entry(P.sched[f], g, line, q);
                outs[f][line * g.L + q] = ((e >> g.logL) << 16) | (e & tmask);
            }
        }
    }
    return PERM_OK;
}

int perm_plan_set_profiling(perm_plan* plan, int enable) {
    if (!plan) return fail(PERM_EINVAL, "null plan");
    plan->profiling = enable != 0;
    return PERM_OK;
}

int perm_plan_set_tracing(perm_plan* plan, int enable) {
    if (!plan) return fail(PERM_EINVAL, "null plan");
    if (!plan->on_device) return fail(PERM_ENODEVICE, "host-only plan");
    if (!enable) {
        cudaFree(plan->d_trace);
        plan->d_trace = nullptr;
        return PERM_OK;
    }
    if (plan->d_trace) return PERM_OK;
    int64_t mx = 1;
    for (int f = 0; f < 3; ++f) {
        const perm::RowPass& rp = plan->host.rp[f];
        mx = std::max<int64_t>(mx, rp.tma ? rp.grid : rp.ctas);
    }
    mx = std::max<int64_t>(mx, plan->host.fused3_grid);
    mx = std::max<int64_t>(mx, plan->host.cluster);
    plan->trace_stride = mx;
    cudaError_t e = cudaMalloc(&plan->d_trace, (size_t)(3 * mx * 16) * sizeof(unsigned long long));
    if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc trace");
    e = cudaMemset(plan->d_trace, 0, (size_t)(3 * mx * 16) * sizeof(unsigned long long));
    if (e != cudaSuccess) return cuda_fail(e, "cudaMemset trace");
    return PERM_OK;
}

int64_t perm_plan_trace(const perm_plan* plan, uint64_t* out, int64_t max_entries) {
    if (!plan) return fail(PERM_EINVAL, "null plan");
    if (!plan->d_trace) return 0;
    const int64_t n = 3 * plan->trace_stride * 16;
    if (out && max_entries > 0) {
        cudaError_t e = cudaMemcpy(out, plan->d_trace, (size_t)std::min(n, max_entries) * 8,
                                   cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpy trace");
    }
    return n;
}

int perm_plan_pass_times(const perm_plan* plan, float* ms, int max_k) {
    if (!plan || !ms) return fail(PERM_EINVAL, "null argument");
    if (!plan->on_device) return fail(PERM_ENODEVICE, "host-only plan");
    const int k = plan->last_kernels;
    if (k <= 0) return 0;
    cudaError_t e = cudaEventSynchronize(plan->ev[k]);
    if (e != cudaSuccess) return cuda_fail(e, "cudaEventSynchronize");
    int w = 0;
    for (int i = 0; i < k && w < max_k; ++i) {
        float t = 0;
        e = cudaEventElapsedTime(&t, plan->ev[i], plan->ev[i + 1]);
        if (e != cudaSuccess) return cuda_fail(e, "cudaEventElapsedTime");
        ms[w++] = t;
    }
    return w;
}

int perm_plan_run_pass(const perm_plan* plan, int32_t pass, const void* in, void* out,
                       perm_stream_t stream) {
    if (!plan) return fail(PERM_EINVAL, "null plan");
    if (!plan->on_device) return fail(PERM_ENODEVICE, "plan was created host-only");
    const HostPlan& P = plan->host;
    if (P.layout != 3 || P.fused3 || plan->d_p || P.r_l)
        return fail(PERM_EUNSUPPORTED, "run_pass needs an unsharded 3-launch TLC plan");
    if (pass < 0 || pass > 2) return fail(PERM_EINVAL, "pass must be 0, 1 or 2");
    if (!in) {
        if (pass == 0) return fail(PERM_EINVAL, "pass 0 needs an input buffer");
        in = plan->d_scratch[pass - 1];        // the plan's own intermediate
    }
    if (pass == 2 && !out) return fail(PERM_EINVAL, "pass 2 needs an output buffer");
    if ((reinterpret_cast<uintptr_t>(in) | reinterpret_cast<uintptr_t>(out)) & 15)
        return fail(PERM_EINVAL, "buffers must be 16-byte aligned");
    uint32_t* dst = pass == 0 ? plan->d_scratch[0] : (pass == 1 ? plan->d_scratch[1] : static_cast<uint32_t*>(out));
    if (overlap(in, dst, P.n * P.eb)) return fail(PERM_EINVAL, "input overlaps the pass output");
    const cudaError_t e = perm::launch_tlc_pass(P, pass, plan->tlc_maps, plan->d_phase[pass],
                                                static_cast<const uint32_t*>(in), dst,
                                                static_cast<cudaStream_t>(stream), true, nullptr);
    if (e != cudaSuccess) return cuda_fail(e, "run_pass launch");
    return PERM_OK;
}

int perm_apply(const perm_plan* plan_c, const void* a, void* b, perm_stream_t stream) {
    perm_plan* plan = const_cast<perm_plan*>(plan_c);   // only profiling bookkeeping mutates
    if (!plan || !a || !b) return fail(PERM_EINVAL, "null plan or buffer");
    if (!plan->on_device) return fail(PERM_ENODEVICE, "plan was created host-only");
    const HostPlan& P = plan->host;
    if (P.r_l) return fail(PERM_EINVAL, "row-sharded plan: use perm_apply_sharded or perm_sharded_step");
    if (overlap(a, b, P.n * P.eb)) return fail(PERM_EINVAL, "a and b overlap (out-of-place only)");
    if ((reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(b)) & 15)
        return fail(PERM_EINVAL, "a and b must be 16-byte aligned");
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const uint32_t* in = static_cast<const uint32_t*>(a);
    uint32_t* out = static_cast<uint32_t*>(b);
    const bool prof = plan->profiling;
    int ev = 0;
    auto mark = [&]() {
        if (prof) cudaEventRecord(plan->ev[ev++], s);
    };
    auto tr = [&](int f) -> unsigned long long* {
        return plan->d_trace ? plan->d_trace + (int64_t)f * plan->trace_stride * 16 : nullptr;
    };
    cudaError_t e = cudaSuccess;
    int k = 0;   // index of the kernel being launched (for the error message)
    mark();
    if (plan->d_p) {
        // low distribution (D_w(P) <= 2n/w, L699-L701): one coalesced kernel; d_p holds
        // q = P^-1 for the S-designated kernel (direct 1) or p for the D-designated (2)
        // or, for whole aligned blocks moved in order (direct 3), qb = block map of P^-1
        e = P.direct == 3   ? perm::launch_block_gather(plan->d_p, in, out, P.n, s)
            : P.direct == 2 ? perm::launch_scatter(plan->d_p, in, out, P.n, 4, s)
                            : perm::launch_gather(plan->d_p, in, out, P.n, 4, s);
        mark();
    } else if (P.passes == 1) {
        const uint32_t* sc[3] = {plan->d_phase[0], plan->d_phase[1], plan->d_phase[2]};
        e = perm::launch_fused(P, sc, in, out, s);
        mark();
    } else if (P.passes == 2) {
        const uint32_t* sc[3] = {plan->d_phase[0], plan->d_phase[1], plan->d_phase[2]};
        e = perm::launch_cluster(P, sc, in, out, s, tr(0));
        mark();
    } else if (P.layout == 3 && P.fused3) {
        const uint32_t* sc[3] = {plan->d_phase[0], plan->d_phase[1], plan->d_phase[2]};
        e = perm::launch_tlc_fused(P, plan->tlc_maps, sc, in, plan->d_scratch[0], plan->d_scratch[1], out,
                                   plan->d_sync, s, tr(0));
        mark();
    } else if (P.layout == 3) {
        uint32_t* x1 = plan->d_scratch[0];
        uint32_t* x2 = plan->d_scratch[1];
        e = perm::launch_tlc_pass(P, 0, plan->tlc_maps, plan->d_phase[0], in, x1, s, false, tr(0));
        mark();
        if (e == cudaSuccess) { ++k; e = perm::launch_tlc_pass(P, 1, plan->tlc_maps, plan->d_phase[1], x1, x2, s, !prof, tr(1)); mark(); }
        if (e == cudaSuccess) { ++k; e = perm::launch_tlc_pass(P, 2, plan->tlc_maps, plan->d_phase[2], x2, out, s, !prof, tr(2)); mark(); }
    } else if (P.layout == 5) {
        // TLC passes through the half-tile ring: a -> X1 -> X2 -> b, chunked tensor stores
        uint32_t* x1 = plan->d_scratch[0];
        uint32_t* x2 = plan->d_scratch[1];
        e = perm::launch_row_pass(P, 0, plan->d_phase[0], in, x1, s, false, tr(0), &plan->tlc_maps[0]);
        mark();
        if (e == cudaSuccess) { ++k; e = perm::launch_row_pass(P, 1, plan->d_phase[1], x1, x2, s, !prof, tr(1), &plan->tlc_maps[1]); mark(); }
        if (e == cudaSuccess) { ++k; e = perm::launch_row_pass(P, 2, plan->d_phase[2], x2, out, s, !prof, tr(2)); mark(); }
    } else if (P.passes == 3) {
        uint32_t* x1 = plan->d_scratch[0];
        uint32_t* x2 = plan->d_scratch[1];
        e = perm::launch_row_pass(P, 0, plan->d_phase[0], in, x1, s, false, tr(0));
        mark();
        if (e == cudaSuccess) { ++k; e = perm::launch_row_pass(P, 1, plan->d_phase[1], x1, x2, s, !prof, tr(1)); mark(); }
        if (e == cudaSuccess) { ++k; e = perm::launch_row_pass(P, 2, plan->d_phase[2], x2, out, s, !prof, tr(2)); mark(); }
    } else {
        uint32_t* x1 = plan->d_scratch[0];
        uint32_t* x2 = plan->d_scratch[1];
        e = perm::launch_row_pass(P, 0, plan->d_phase[0], in, x1, s, false, tr(0));
        mark();
        if (e == cudaSuccess) { ++k; e = perm::launch_transpose(x1, x2, P.r, P.c, s, !prof); mark(); }
        if (e == cudaSuccess) { ++k; e = perm::launch_row_pass(P, 1, plan->d_phase[1], x2, x1, s, !prof, tr(1)); mark(); }
        if (e == cudaSuccess) { ++k; e = perm::launch_transpose(x1, x2, P.c, P.r, s, !prof); mark(); }
        if (e == cudaSuccess) { ++k; e = perm::launch_row_pass(P, 2, plan->d_phase[2], x2, out, s, !prof, tr(2)); mark(); }
    }
    if (e != cudaSuccess) {
        if (prof) plan->last_kernels = 0;
        return cuda_fail(e, ("launch of kernel " + std::to_string(k) + " of " +
                             std::to_string(P.passes)).c_str());
    }
    if (prof) plan->last_kernels = ev - 1;
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "kernel launch");
    return PERM_OK;
}

namespace {
int apply_host_impl(perm_plan* plan, const void* a_host, void* b_host, perm_stream_t stream, bool sync) {
    if (!plan || !a_host || !b_host) return fail(PERM_EINVAL, "null plan or buffer");
    if (!plan->on_device) return fail(PERM_ENODEVICE, "plan was created host-only");
    if (plan->host.r_l) return fail(PERM_EINVAL, "row-sharded plan: use perm_apply_sharded or perm_sharded_step");
    const size_t bytes = (size_t)plan->host.n * plan->host.eb;
    cudaError_t e;
    if (!plan->d_stage[0]) {
        for (int i = 0; i < 2; ++i) {
            e = cudaMalloc(&plan->d_stage[i], bytes);
            if (e != cudaSuccess) return fail(PERM_ENOMEM, std::string("cudaMalloc staging: ") + cudaGetErrorString(e));
        }
    }
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    e = cudaMemcpyAsync(plan->d_stage[0], a_host, bytes, cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpyAsync H2D");
    int st = perm_apply(plan, plan->d_stage[0], plan->d_stage[1], stream);
    if (st != PERM_OK) return st;
    e = cudaMemcpyAsync(b_host, plan->d_stage[1], bytes, cudaMemcpyDeviceToHost, s);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpyAsync D2H");
    if (sync) {
        e = cudaStreamSynchronize(s);
        if (e != cudaSuccess) return cuda_fail(e, "cudaStreamSynchronize");
    }
    return PERM_OK;
}
}  // namespace

int perm_apply_host(perm_plan* plan, const void* a_host, void* b_host, perm_stream_t stream) {
    return apply_host_impl(plan, a_host, b_host, stream, true);
}

int perm_apply_host_async(perm_plan* plan, const void* a_host, void* b_host, perm_stream_t stream) {
    return apply_host_impl(plan, a_host, b_host, stream, false);
}

int perm_scatter_baseline(const int32_t* p_dev, const void* a, void* b, int64_t n,
                          int32_t elem_bytes, perm_stream_t stream) {
    if (!p_dev || !a || !b || n <= 0) return fail(PERM_EINVAL, "null argument or n <= 0");
    if ((elem_bytes != 4 && elem_bytes != 8) || (n & 3))
        return fail(PERM_EUNSUPPORTED, "elem_bytes 4 or 8, n % 4 == 0");
    cudaError_t e = perm::launch_scatter(p_dev, a, b, n, elem_bytes, static_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "scatter launch");
    return PERM_OK;
}

int perm_gather_baseline(const int32_t* q_dev, const void* a, void* b, int64_t n,
                         int32_t elem_bytes, perm_stream_t stream) {
    if (!q_dev || !a || !b || n <= 0) return fail(PERM_EINVAL, "null argument or n <= 0");
    if ((elem_bytes != 4 && elem_bytes != 8) || (n & 3))
        return fail(PERM_EUNSUPPORTED, "elem_bytes 4 or 8, n % 4 == 0");
    cudaError_t e = perm::launch_gather(q_dev, a, b, n, elem_bytes, static_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "gather launch");
    return PERM_OK;
}

int perm_copy_kernel(const void* a, void* b, int64_t n, int32_t elem_bytes, perm_stream_t stream) {
    if (!a || !b || n <= 0) return fail(PERM_EINVAL, "null argument or n <= 0");
    const int64_t words = n * elem_bytes / 4;
    if (words & 3) return fail(PERM_EUNSUPPORTED, "n*elem_bytes must be a multiple of 16");
    cudaError_t e = perm::launch_copy(static_cast<const uint32_t*>(a), static_cast<uint32_t*>(b),
                                      words, static_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return cuda_fail(e, "copy launch");
    return PERM_OK;
}

int perm_last_error(void) { return g_status; }
const char* perm_last_error_string(void) { return g_msg.c_str(); }
const char* perm_version(void) { return "libperm 0.1 (sm_100a)"; }

}  // extern "C"
