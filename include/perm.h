/*
 * perm.h — C ABI of libperm, the B200 (sm_100a) offline permutation library.
 *
 * Operation (§IV): given a permutation P of {0..n-1}, stored in
 * an int32 array p with p[i] = P(i) and known in advance ("offline"), copy
 * a[i] to b[P(i)] for every i. The result is unique; libperm produces it
 * bit-exactly (raw 4-byte words are moved, never interpreted as floats).
 *
 * Method (§V-§VII, Thm 9): view a and b as r x c matrices and
 * apply a row-wise permutation, a column-wise permutation (= transpose,
 * row-wise, transpose; Lemma 8) and a row-wise permutation. The three
 * per-line permutations come from a König edge-colouring of the row-level
 * bipartite multigraph (L537-L539, L603-L605); every shared-memory permute
 * hop is bank-conflict-free because of a second colouring of each line's
 * bank-level graph (Thm 6). Both colourings are computed
 * once per P on the host by perm_plan_create (the "offline" cost, timed and
 * reported separately); perm_apply is the data-parallel hot path.
 *
 * Thread safety: distinct plans may be used from distinct threads. A plan
 * is immutable after creation, but it owns scratch buffers, so at most ONE
 * perm_apply may be in flight per plan at a time (use one plan per stream).
 * Error status is thread-local (perm_last_error).
 */
#ifndef LIBPERM_PERM_H
#define LIBPERM_PERM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* cudaStream_t is passed as an opaque pointer so this header does not need
 * the CUDA headers; NULL means the legacy default stream. */
typedef void* perm_stream_t;

typedef struct perm_plan perm_plan;   /* opaque */

enum perm_status {
    PERM_OK           =  0,
    PERM_EINVAL       = -1,  /* null pointer, n <= 0, a == b / overlapping buffers, bad option */
    PERM_ENOTPERM     = -2,  /* p is not a permutation of 0..n-1 (value out of range or repeated) */
    PERM_EUNSUPPORTED = -3,  /* n not a power of two in [2^10, 2^30] (2^9..2^29 for 8-byte
                                elements), or elem_bytes not 4 or 8 */
    PERM_ENOMEM       = -4,  /* host or device allocation failed */
    PERM_ECUDA        = -5,  /* a CUDA runtime call failed (message has the CUDA error) */
    PERM_ENCCL        = -6,  /* NCCL missing or an NCCL call failed (row-sharded path) */
    PERM_ENODEVICE    = -7   /* the call needs a device but the plan is host-only / no GPU */
};

/* Pass structures a plan may use (perm_plan_info.passes). */
enum perm_passes {
    PERM_PASSES_AUTO  = 0,
    PERM_PASSES_FUSED = 1,   /* n <= 2^14: all three phases inside one CTA's shared memory */
    PERM_PASSES_CLUSTER = 2, /* n = 2^15..2^18 (default 2^15..2^17): ONE launch; the array lives in the shared memory
                                of one thread-block cluster (2..16 blocks); the column phase's
                                two transposes become block exchanges over distributed shared
                                memory (DSMEM bulk copies); a and b cross HBM once each */
    PERM_PASSES_3     = 3,   /* R1, R2, R3; both transposes absorbed into tiled layouts */
    PERM_PASSES_5     = 5    /* R, T, R, T, R: the paper's five kernel calls (L699) */
};

/* Intermediate layouts of the 3-pass pipeline (perm_plan_options.layout). */
enum perm_layout {
    PERM_LAYOUT_AUTO  = 0,
    PERM_LAYOUT_TILED = 1,   /* reader transposes: X1, X2 stored as h1 x h2 / h3 x h2 tiles */
    /* 2 (LINES) was removed in round 2 */
    PERM_LAYOUT_TLC   = 3,   /* tile-level colouring: the transposes absorbed into the passes'
                                X1 / X2 chunk layouts (default 2^18..2^25) */
    PERM_LAYOUT_TLC_RING = 5 /* TLC with 32768-word tiles permuted in place through the
                                half-tile ring (3 passes at 2^26 / 2^27; measured slower than
                                the 5-pass default there, kept as an option) */
};

typedef struct {
    int32_t passes;      /* enum perm_passes; 0 = choose by n */
    int32_t h1, h2, h3;  /* lines per CTA tile in the three row passes; 0 = choose */
    int32_t layout;      /* enum perm_layout; 0 = choose by n */
    int32_t stages;      /* TMA pipeline depth of the LINES layout (0 = as many as fit, <= 4) */
    int32_t fuse;        /* LINES layout, square view: 1 = run the three passes as ONE persistent
                            kernel with grid barriers; 0 = auto (currently three launches
                            chained with programmatic dependent launch); -1 = never */
    int32_t no_tma;      /* 1: use the plain (non-TMA) row-pass kernels of the 5-pass / sharded
                            structures even when a TMA stage fits (testing, A/B comparisons);
                            -1: TMA slots hold the data only and the schedule is read from global
                            memory (the default wherever a line + its schedule exceed a slot:
                            L >= 16384, n >= 2^27) */
    int32_t direct;      /* low-distribution shortcut (for P with
                            D_w(P) <= 2n/w, e.g. identical and shuffle, a one-kernel copy
                            is coalesced and faster): 0 = auto (on when D_w(P) <= 2n/32),
                            -1 = never (always run the scheduled passes), 1 = always, with
                            the S-designated kernel b[i] = a[q[i]], q = P^-1 (L373; writes
                            whole sectors, reads D_w(P^-1) = D_w(P) groups), 2 = always,
                            with the D-designated kernel b[p[i]] = a[i] (L365). Auto (0) runs
                            a block gather instead (info.direct = 3) when P moves whole aligned
                            32-word blocks in order (p[32j + x] = 32g + x: the identical
                            permutation, block permutations), reading n/32 block indices */
    int32_t log2c;       /* view r x c with c = 2^log2c (the view "is not
                            restricted to a square matrix"); 0 = c = 2^ceil(k/2) */
    int32_t sched_format; /* TLC layout entry format: -1 = full (source row << log2(tile) |
                             destination); 1 = compact (the line index inside the tile is implied
                             by the source offset: 19 instead of 21 bits at n = 2^22) wherever a
                             kernel is compiled for its width (not with fuse = 1); 0 = compact
                             from n = 2^23 on, full below (measured).
                             5-pass per-line schedules: 0 = dense bitstreams (E bits per entry)
                             for lines of 16384 words (the schedule-from-global slots), W64
                             elsewhere; 2 = dense for every line length; -1 = W64 everywhere */
    int32_t gpu_planner; /* where the offline colourings run: 1 = on the
                            current CUDA device (gplan.cu: Euler split with ruling-set cycle
                            labelling), -1 = host threads (planner.cpp), 0 = auto (device for
                            device plans with n >= 2^20, host otherwise) */
    int32_t cluster;     /* cluster path (passes = 2): thread blocks per cluster, a power of two
                            in 2..16; 0 = 16 (raised never; a block must hold 2048..16384 words) */
} perm_plan_options;

typedef struct {
    int64_t n;
    int64_t rows, cols;          /* the r x c view (L603) */
    int64_t sched_bytes;         /* device bytes of the three packed bank schedules */
    int64_t scratch_bytes;       /* device bytes of intermediate buffers */
    int32_t elem_bytes;
    int32_t passes;              /* 1, 2 (cluster), 3 or 5; 0 for a low-distribution shortcut plan
                                    (direct != 0: one kernel, no schedule) */
    int32_t kernels_per_apply;   /* kernel launches one perm_apply issues */
    int32_t entry_bits[3];       /* bits per schedule entry, phase 1..3 (2*log2(L) - 5) */
    int32_t h[3];                /* lines per CTA of the three row passes */
    int32_t planner_threads;     /* OpenMP threads the planner used */
    double  build_ms_colour;     /* row-level König colouring (Euler split) */
    double  build_ms_bank;       /* per-line bank-level colourings + packing */
    double  build_ms_upload;     /* device allocation + host->device copy */
    int32_t world, rank;         /* row sharding (1, 0 for unsharded plans) */
    int64_t shard_elems;         /* n / world */
    int64_t block_elems;         /* n / world^2: one all-to-all block */
    int64_t distribution;        /* D_w(P), w = 32 (L389-L401): address groups the warps write */
    int32_t direct;              /* 1: perm_apply runs the S-designated kernel on q = P^-1,
                                    2: the D-designated kernel on p (low D_w), 3: the block
                                    gather on P^-1's block map; 0: the scheduled passes */
    int32_t gpu_planner;         /* 1: the colourings ran on the GPU (gplan.cu), 0: on the host */
} perm_plan_info;

/* ------------------------------------------------------------------ plans */

/* Build a plan for P on the CURRENT CUDA device: validates p (O(n) bitmap),
 * colours, packs and uploads the schedules and allocates scratch.
 * p: host int32[n], borrowed for the duration of the call only.
 * n: power of two, 2^10 <= n <= 2^30. elem_bytes: 4, or 8 (n <= 2^29): an 8-byte
 * element moves as a pair of 4-byte words (the word permutation 2P(i)+h is
 * scheduled; info/export then describe 2n words).
 * Returns NULL on error (see perm_last_error). Synchronous. */
perm_plan* perm_plan_create(const int32_t* p, int64_t n, int32_t elem_bytes);

/* Same with explicit options (NULL = defaults). */
perm_plan* perm_plan_create_ex(const int32_t* p, int64_t n, int32_t elem_bytes,
                               const perm_plan_options* opt);

/* Planner only: builds the host-side plan (colourings, packed schedules) and
 * touches no CUDA API. Usable on a machine without a GPU for perm_plan_export
 * and perm_plan_get_info; perm_apply on it returns PERM_ENODEVICE. */
perm_plan* perm_plan_create_host(const int32_t* p, int64_t n, int32_t elem_bytes,
                                 const perm_plan_options* opt);

/* Frees host and device memory. NULL is a no-op. The caller must ensure no
 * perm_apply on this plan is still running on the device. */
void perm_plan_destroy(perm_plan* plan);

int perm_plan_get_info(const perm_plan* plan, perm_plan_info* out);

/* Human/machine-readable JSON description of the plan's pass structure
 * (views, per-pass lines per CTA, threads, elements per thread, shared-memory
 * stride, simulated bank-conflict wavefronts, I/O layouts). Writes at most
 * len bytes including the terminating NUL; returns the full length needed. */
int64_t perm_plan_describe(const perm_plan* plan, char* buf, int64_t len);

/* Export the plan in LOGICAL order for an independent checker:
 *   kappa[x], x in [0,n): row-level colour of element x (uint16; c <= 2^15);
 *   sched1[i*c + q], sched2[k*r + q], sched3[i*c + q]: for line i (rows for
 *   phases 1 and 3, columns k for phase 2) and slot q = round*32 + lane,
 *   the entry (sigma << 16) | t: the slot reads source s = 32*sigma + lane
 *   and writes destination t.
 * Any output pointer may be NULL to skip it. Host memory, caller-owned. */
int perm_plan_export(const perm_plan* plan, uint16_t* kappa,
                     uint32_t* sched1, uint32_t* sched2, uint32_t* sched3);

/* ------------------------------------------------------------------ apply */

/* b[P(i)] = a[i] for all i. a, b: DEVICE pointers to n*elem_bytes bytes on the
 * plan's device, 16-byte aligned, not overlapping (the algorithm is
 * out-of-place, L361). Asynchronous and stream-ordered: no host sync, no
 * allocation. Launch errors are returned immediately (PERM_ECUDA); device
 * faults surface at the caller's next synchronisation. */
int perm_apply(const perm_plan* plan, const void* a, void* b, perm_stream_t stream);

/* End-to-end variant with HOST buffers: copies a_host to the device, applies,
 * copies the result to b_host, then synchronises the stream. The first call
 * allocates 2*n*elem_bytes of device staging owned by the plan. Pinned host
 * memory gives asynchronous copies; pageable memory works but is slower. */
int perm_apply_host(perm_plan* plan, const void* a_host, void* b_host, perm_stream_t stream);

/* perm_apply_host without the final synchronisation: the H2D copy, the apply and the D2H
 * copy are only enqueued on `stream`, so applies of DIFFERENT plans on different streams
 * overlap one plan's device->host copy with the next one's host->device copy (the copy
 * engines of the two directions run concurrently). a_host / b_host must be pinned, must
 * stay valid and a_host unmodified until the stream is synchronised, and b_host holds the
 * result only after that. The plan's staging buffers are reused by every call: two calls
 * on the SAME plan must be on the same stream. Errors as perm_apply_host; device faults
 * surface at the caller's synchronisation. */
int perm_apply_host_async(perm_plan* plan, const void* a_host, void* b_host, perm_stream_t stream);

/* Per-kernel timing: when enabled, perm_apply records a CUDA event before its
 * first kernel and after each kernel on the launch stream. perm_plan_pass_times
 * waits for the last event and writes up to max_k kernel durations (ms) of the
 * most recent apply; returns the number written or a negative status. */
int perm_plan_set_profiling(perm_plan* plan, int enable);
int perm_plan_pass_times(const perm_plan* plan, float* ms, int max_k);

/* Tracing (diagnostics): when enabled, every CTA of the three row passes
 * records up to 16 %globaltimer stamps (ns) at its phase boundaries (start,
 * after griddepcontrol.wait, per tile: data ready / permuted / stored, end).
 * perm_plan_trace copies [pass][cta][16] stamps of the most recent apply to
 * host memory (synchronous) and returns the number of entries (3*ctas*16). */
int     perm_plan_set_tracing(perm_plan* plan, int enable);
int64_t perm_plan_trace(const perm_plan* plan, uint64_t* out, int64_t max_entries);

/* Diagnostics (kernel roofline timing): launch ONE row pass of a 3-launch TLC plan
 * (layout 3, not fused, not on the low-distribution shortcut), stream-ordered:
 *   pass 0: in (n words, row-major a)      -> the plan's internal X1
 *   pass 1: in (n words, X1 layout)        -> the plan's internal X2
 *   pass 2: in (n words, X2 layout)        -> out (n words, row-major b)
 * `in` need not come from the previous pass (any data times the same: the
 * schedule, not the data, decides every address); in = NULL for passes 1 and 2
 * reads the plan's own X1 / X2, so run_pass(0, a), (1, NULL), (2, NULL, b) is
 * perm_apply. PERM_EUNSUPPORTED for other plans. */
int perm_plan_run_pass(const perm_plan* plan, int32_t pass, const void* in, void* out,
                       perm_stream_t stream);

/* ------------------------------------------------- row-sharded (multi-GPU) */

/* rank g of `world` GPUs owns rows [g*r/world, (g+1)*r/world) of the
 * r x c view, i.e. the contiguous shard a[g*n/world : (g+1)*n/world] (and the
 * same shard of b). Phases 1 and 3 (row-wise, L537-L539) are local; the
 * column-wise phase (Lemma 8: transpose, row-wise, transpose) becomes two
 * uniform, P-independent all-to-all exchanges of n/world^2-element blocks over
 * NCCL (NVLink / NVSwitch). p is the FULL permutation (every rank passes the
 * same p; every rank colours it identically and keeps its own lines' schedules).
 * world must be a power of two with r/world >= 32 and c/world >= 32. */

#define PERM_NCCL_UID_BYTES 128

/* Writes a fresh ncclUniqueId (PERM_NCCL_UID_BYTES bytes, host memory) to uid_out.
 * Rank 0 calls it and broadcasts the bytes to the other ranks out of band (e.g.
 * torch.distributed). NCCL is loaded at run time (the process's libnccl.so.2);
 * PERM_ENCCL when it cannot be loaded. */
int perm_nccl_unique_id(void* uid_out);

/* Sharded plan of rank `rank` on the CURRENT device. nccl_uid (PERM_NCCL_UID_BYTES
 * bytes, the same on every rank; borrowed for the call) != NULL: the call also
 * joins an NCCL communicator of `world` ranks (collective: every rank must call
 * it concurrently; it blocks until all have joined) and allocates the plan's two
 * exchange shards (2 * n/world * elem_bytes device bytes), so perm_apply_sharded
 * works. nccl_uid == NULL: no communicator; only perm_sharded_step is available
 * (the caller runs the exchanges, e.g. virtual ranks on one GPU).
 * NULL on error: PERM_EINVAL / PERM_EUNSUPPORTED as perm_plan_create, or
 * PERM_ENCCL when NCCL cannot be loaded or the communicator fails. */
perm_plan* perm_plan_create_sharded(const int32_t* p, int64_t n, int32_t elem_bytes,
                                    int32_t world, int32_t rank, const void* nccl_uid);
perm_plan* perm_plan_create_sharded_ex(const int32_t* p, int64_t n, int32_t elem_bytes,
                                       int32_t world, int32_t rank, const void* nccl_uid,
                                       const perm_plan_options* opt);
/* Planner only (no CUDA, no NCCL): for perm_plan_export / perm_plan_get_info. */
perm_plan* perm_plan_create_sharded_host(const int32_t* p, int64_t n, int32_t elem_bytes,
                                         int32_t world, int32_t rank,
                                         const perm_plan_options* opt);

/* The whole sharded apply on this rank: b_shard = rows [rank*r/world, ...) of b,
 * b[P(i)] = a[i]. a_shard, b_shard: DEVICE buffers of n/world elements on the
 * plan's device, 16-byte aligned, not overlapping. Stream-ordered, no host sync:
 *   step 0 -> all-to-all -> step 1 -> all-to-all -> step 2
 * with the plan's own exchange shards; every rank must call it (NCCL collective).
 * PERM_ENCCL if the plan has no communicator; at most one in flight per plan. */
int perm_apply_sharded(const perm_plan* plan, const void* a_shard, void* b_shard,
                       perm_stream_t stream);

/* One local step of a sharded apply (device buffers, stream-ordered):
 *   step 0: in = a shard (n/world elems)  -> out = send buffer (n/world)  [R1 (+ T)]
 *   step 1: in = recv buffer              -> out = send buffer            [R2 (+ T)]
 *   step 2: in = recv buffer              -> out = b shard                [R3]
 * For n = 2^15..2^25 words (TLC form, info.passes == 3) each step is ONE tile-coloured pass
 * that writes the send buffer in the exchange layout directly; beyond (per-line form,
 * info.passes == 5) steps 0 and 1 are a row pass plus a transpose. The buffers' contents
 * differ between the forms; the block contract below is the same.
 * Between steps 0->1 and 1->2 the caller performs the all-to-all: with
 * B = n/world^2, for every pair (g, q): recv_q[g*B : (g+1)*B] = send_g[q*B : (q+1)*B]
 * (perm_sharded_exchange, or device copies for ranks sharing one GPU). */
int perm_sharded_step(const perm_plan* plan, int32_t step, const void* in, void* out,
                      perm_stream_t stream);

/* The all-to-all of the step contract above on the plan's NCCL communicator
 * (grouped ncclSend / ncclRecv, one pair per peer), stream-ordered. send, recv:
 * DEVICE buffers of n/world elements. PERM_ENCCL without a communicator. */
int perm_sharded_exchange(const perm_plan* plan, const void* send, void* recv,
                          perm_stream_t stream);

/* ------------------------------------------------------- comparators */

/* D-designated (conventional) algorithm: b[p[i]] = a[i] in one
 * kernel. p_dev: DEVICE int32[n] (a valid permutation; not checked). */
int perm_scatter_baseline(const int32_t* p_dev, const void* a, void* b, int64_t n,
                          int32_t elem_bytes, perm_stream_t stream);

/* S-designated algorithm: b[i] = a[q[i]], q = P^{-1} (DEVICE). */
int perm_gather_baseline(const int32_t* q_dev, const void* a, void* b, int64_t n,
                         int32_t elem_bytes, perm_stream_t stream);

/* Plain device-to-device copy of n*elem_bytes with the same vectorised
 * kernel style (the identity lower bound used for roofline context). */
int perm_copy_kernel(const void* a, void* b, int64_t n, int32_t elem_bytes,
                     perm_stream_t stream);

/* ------------------------------------------------------------- status */

int         perm_last_error(void);          /* thread-local status of the last failed call */
const char* perm_last_error_string(void);   /* thread-local message, never NULL */
const char* perm_version(void);

#ifdef __cplusplus
}
#endif
#endif /* LIBPERM_PERM_H */
