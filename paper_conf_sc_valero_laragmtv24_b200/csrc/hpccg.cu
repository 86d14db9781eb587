// hpccg.cu -- C ABI (include/hpccg.h) and host orchestration of the B200
// HPCCG CG hot path: contexts, on-device problem generation, the halo
// exchange (NCCL or loopback), and the CG solve loop replayed as a CUDA graph
// with every scalar kept on the device.  Design: DESIGN.md.
#include <cuda_runtime.h>
#include <math.h>
#include <stdarg.h>
#include <stdlib.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <string>
#include <unordered_map>
#include <utility>
#include <vector>

#include "hpccg.h"
#include "kernels.cuh"
#include "tridiag.cuh"
#include "lbm.cuh"

#ifdef HPCCG_WITH_NCCL
#include <nccl.h>
#endif

using namespace hpccg;

namespace {

thread_local std::string g_err;

int fail(int code, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return code;
}

#define CU(call)                                                                       \
    do {                                                                               \
        cudaError_t e_ = (call);                                                       \
        if (e_ != cudaSuccess)                                                         \
            return fail(HPCCG_ECUDA, "%s failed: %s (%s:%d)", #call,                   \
                        cudaGetErrorString(e_), __FILE__, __LINE__);                   \
    } while (0)

#define CHECK(expr)                        \
    do {                                   \
        int rc_ = (expr);                  \
        if (rc_ != HPCCG_OK) return rc_;   \
    } while (0)

enum Mode { MODE_SINGLE = 0, MODE_NCCL = 1, MODE_LOOPBACK = 2, MODE_PEER = 3 };
enum Phase { PH_PUPDATE = 0, PH_SPMV, PH_UPDATE, PH_ALLREDUCE, PH_EXCHANGE, PH_N };

int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Blocks needed for `work` thread-units, capped at one resident wave
// (SM count x blocks per SM from the occupancy calculator).
int wave_grid(int64_t work, int wave) {
    int64_t b = cdiv(std::max<int64_t>(work, 1), kBlock);
    return (int)std::max<int64_t>(1, std::min<int64_t>(b, wave));
}

bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

}  // namespace

// ------------------------------------------------------------------ structs

struct hpccg_ctx {
    int device = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    cudaStream_t comm_stream = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    int rank = 0, nranks = 1, nslabs = 1;
    Mode mode = MODE_SINGLE;
    // BLAS-1 kernels: 16-B units per thread per trip (2 or 4), tuned on B200 at
    // n = 1e9: AXPY 2 (6.67 TB/s; 4: 6.28), DOT 4 (7.05; 2: 6.75)
    int axpy_unroll = 2, dot_unroll = 4;
#ifdef HPCCG_WITH_NCCL
    ncclComm_t comm = nullptr;
#endif
    // scratch for the API reductions (ddot / maxabsdiff): per slab loc / out
    double *d_api = nullptr;             // [2 * nslabs]: loc[s], out[s]
    double **d_api_src = nullptr;        // loopback allreduce tables
    double **d_api_dst = nullptr;
    Reduction red{};                     // partials + counter
    int64_t red_cap = 0;
    double *h_pinned = nullptr;          // 8 doubles, pinned + mapped
    double *d_mapped = nullptr;          // device alias of h_pinned (zero-copy result)
    int64_t launches = 0;
    int num_sms = 148;
    int max_persist_l2 = 0, max_window = 0;  // bytes (device attributes)
    int max_cluster = 0;                     // CTAs of the one-cluster persistent solve
    int smem_cluster = 0;                    // CTAs of the shared-memory-resident solve
    int64_t smem_bytes = 0;                  // dynamic smem per CTA it may use
    std::unordered_map<const void *, int> occ;  // kernel -> resident blocks / SM
};

struct Slab {
    int rank = 0;
    int64_t n = 0, plane = 0, ncol = 0;
    unsigned long long nnz = 0;
    double *val = nullptr;
    int *col = nullptr;
    double *b = nullptr, *x = nullptr, *xexact = nullptr, *r = nullptr, *Ap = nullptr;
    double *p_alloc = nullptr, *p = nullptr;  // p: local-with-halo base (ncol)
    // r, x, Ap and p live in one contiguous "arena" so one L2 access-policy
    // window can keep the CG vectors resident
    double *arena = nullptr;
    size_t arena_bytes = 0;
    CgScalars *sc = nullptr;
    Reduction red{};
    unsigned *bar = nullptr;  // grid barrier state of the persistent solve
    TraceSlot *trace = nullptr;  // HPCCG_OPT_TRACE buffer: [trace_max][3]
    int trace_max = 0;
    bool trace_on = false;
    double *spmv_parts = nullptr;  // per-block p.Ap partials (single slab); f2: 2 arrays
    int64_t spmv_nparts = 0;
    double *sv = nullptr;  // f2 single-reduction CG: s = A p recurrence vector (n)
    PeerSync *psync = nullptr;  // HALO_PEER: this slab's flags / allreduce slots
    PeerTab *ptab = nullptr;    // HALO_PEER: device copy of the peer table
    int early_trigger = 1;      // HPCCG_OPT_PDL 1: SpMV triggers its successor early
    int nx = 0;                 // grid row stride (DIA-27 column formation)
    int dia = 0;                // HPCCG_OPT_SPMV_FORMAT 1: DIA-27 SpMV (col[] not read)
    unsigned char *sl = nullptr;  // HPCCG_OPT_SPMV_SLICED: chunk-sliced copy of the ELL (324 B per row)
    // HPCCG_OPT_FUSE_PSPMV: ticket counter, error word, per-chunk flags
    unsigned char *ps_mem = nullptr;
    unsigned *ps_ticket = nullptr;
    unsigned long long *ps_flags = nullptr;
    int *ps_err = nullptr;
    // HPCCG_OPT_DEFER_X = m >= 2: ring slots 1..pring_slots of p (slot 0 = p),
    // each laid out like p (halo base, ncol), pring_stride doubles apart
    double *pring_alloc = nullptr, *pring = nullptr;
    int64_t pring_stride = 0;
    int pring_slots = 0;
};

struct TimedOp {
    int phase;
    cudaEvent_t a, b;
};

struct hpccg_problem {
    hpccg_ctx *ctx = nullptr;
    int nx = 0, ny = 0, nz = 0;
    std::vector<Slab> slabs;
    unsigned long long nnz_global = 0;
    int64_t red_cap = 0;  // partial slots per slab reduction scratch
    // loopback allreduce tables (device arrays of device pointers)
    double **d_tab = nullptr;  // [8][nslabs]: src/dst pAp, src/dst rr, src/dst red, src/dst gd (f2)
    // options
    int opt_graph = 1, opt_poll = 8, opt_timing = 0, opt_minb = 0, opt_while = 1, opt_l2 = 1;
    int opt_vec_waves = 1;  // 0: one thread per double2 (full grid); k: k resident waves
    int opt_rows = 2;       // SpMV rows per thread (2 when aligned, else 1)
    int opt_unroll = 4;     // CG vector kernels: 16-B units per thread per trip
    int opt_persist = 1;    // 0 never, 1 auto (see opt_persist_rows), 2 always (single slab)
    int opt_pdl = 1;        // programmatic dependent launch between the CG kernels
    // auto threshold: -1 (default) = only when the on-chip (shared-memory) solve fits --
    // the while-graph beats the grid / one-cluster persistent solves at every size
    // above that; k >= 0 = when n <= k
    int64_t opt_persist_rows = -1;
    int64_t opt_cluster_rows = 16384;  // persistent solve as one cluster up to this many rows
    int opt_smem = 1;                  // persistent solve resident in cluster shared memory if it fits
    int opt_while_unroll = 4;          // CG iterations per WHILE-body execution
    int opt_variant = 0;               // 0 HPCCG CG, 1 single-reduction CG (f2)
    int opt_ff = 1;                    // single slab: finisher-free HPCCG loop (consumer-side sums)
    int opt_serp = -1;                 // HPCCG_OPT_SERPENTINE bit mask (-1 auto)
    // HALO_PEER = 2, per slab: ((grid, unroll) key, blocks of the p update that push a plane)
    std::vector<std::pair<uint64_t, unsigned>> fpush;
    int opt_smem_threads = 0;          // on-chip solve CTA width: 0 auto, 256, 512
    int opt_peer = 0;                  // multi-slab: halo push + allreduce over peer memory
    int64_t opt_peer_timeout_ms = 30000;  // give up a peer-memory wait after this long
    int opt_defer_x = -1;              // finisher-free loop: x update deferred into the p update (-1 auto,
                                       // 0 off, 1 every iteration, m >= 2 over a ring of m + 1 p buffers)
    int opt_fuse_ps = 0;               // p update + SpMV in one pipelined kernel (-1 auto, 0 off, 1 on)
    int opt_spmv_trips = 1;            // single-slab SpMV trips per block (0 auto, 1 off, T)
    int opt_pap_cluster = 0;           // p.Ap finisher as one 8-CTA cluster (1) or one CTA (0)
    int opt_sliced = 0;                // CG SpMV from the chunk-sliced copy via TMA (-1 auto, 0, 1)
    int opt_smem_halo = -1;            // on-chip solve: gathered vector halo'd in every CTA (-1 auto, 0, 1)
    int opt_spmv_cl = 0;               // CG SpMV in 8-CTA clusters, one p.Ap partial per cluster (-1 auto, 0, 1)
    int opt_ps_lead = 0;               // its production lead in chunks (0: plane / 512 + 8)
    std::vector<void *> ipc_opened;    // peers' buffers mapped with cudaIpcOpenMemHandle
    bool peer_ring = false;            // the peer tables address the neighbours' p rings
    int last_persist_mode = 3;
    // graph of one CG iteration (per-iteration replay) ...
    cudaGraphExec_t graph = nullptr;
    int64_t graph_kernels = 0;
    // ... or of the whole solve: init + while(!done) { iteration }
    cudaGraphExec_t wgraph = nullptr;
    cudaGraphConditionalHandle whandle = 0;
    int wgraph_max_iter = -1;
    double wgraph_tol = -1.0;
    int64_t wgraph_init_kernels = 0, wgraph_body_kernels = 0;
    bool while_failed = false;
    // timing
    std::vector<cudaEvent_t> ev_pool;
    size_t ev_used = 0;
    std::vector<TimedOp> timed;
    cudaEvent_t ev_t0 = nullptr, ev_t1 = nullptr;
    int *h_done = nullptr;  // pinned poll flags [2]
    CgScalars *h_sc = nullptr;  // pinned copy of slab 0's scalars at the end of a solve
    cudaEvent_t ev_poll[2] = {nullptr, nullptr};
    hpccg_stats stats{};
};

namespace {

#ifdef HPCCG_WITH_NCCL
int nccl_fail(hpccg_ctx *ctx, ncclResult_t r, const char *what) {
    if (ctx->comm) {
        ncclCommAbort(ctx->comm);
        ctx->comm = nullptr;
    }
    return fail(HPCCG_ENCCL, "%s failed: %s", what, ncclGetErrorString(r));
}
#define NC(ctx, call)                                               \
    do {                                                            \
        ncclResult_t r_ = (call);                                   \
        if (r_ != ncclSuccess) return nccl_fail((ctx), r_, #call);  \
    } while (0)
#endif

int check_launch(hpccg_ctx *ctx, int nkernels = 1) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return fail(HPCCG_ECUDA, "kernel launch failed: %s", cudaGetErrorString(e));
    ctx->launches += nkernels;
    return HPCCG_OK;
}

// Launch with optional programmatic dependent launch (PDL): the kernel may be
// scheduled while its stream predecessor drains; it calls pdl_wait() before
// touching anything that predecessor writes (kernels.cuh).
template <typename... KArgs, typename... Args>
cudaError_t launch_kb(bool pdl, void (*kernel)(KArgs...), dim3 grid, dim3 block, cudaStream_t st,
                      Args &&...args) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = 0;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = pdl ? at : nullptr;
    cfg.numAttrs = pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

template <typename... KArgs, typename... Args>
cudaError_t launch_k(bool pdl, void (*kernel)(KArgs...), dim3 grid, cudaStream_t st, Args &&...args) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = grid;
    cfg.blockDim = dim3(kBlock);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = pdl ? at : nullptr;
    cfg.numAttrs = pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

// the p.Ap finisher of a slab whose SpMV left more than kUpdSumMax partials:
// one 1024-thread CTA, or (HPCCG_OPT_PAP_CLUSTER) a cluster of kPapCl CTAs
int launch_pap_finish(hpccg_ctx *ctx, int cluster, const double *parts, unsigned np, CgScalars *sc, bool pdl) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(cluster ? kPapCl : 1);
    cfg.blockDim = dim3(1024);
    cfg.stream = ctx->stream;
    cudaLaunchAttribute at[2];
    int na = 0;
    if (pdl) {
        at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[na++].val.programmaticStreamSerializationAllowed = 1;
    }
    if (cluster) {
        at[na].id = cudaLaunchAttributeClusterDimension;
        at[na].val.clusterDim.x = kPapCl;
        at[na].val.clusterDim.y = 1;
        at[na++].val.clusterDim.z = 1;
    }
    cfg.attrs = na ? at : nullptr;
    cfg.numAttrs = na;
    void (*fk)(const double *, unsigned, CgScalars *) = cluster ? cg_pap_finish_cl_kernel : cg_pap_finish_kernel;
    const cudaError_t e = cudaLaunchKernelEx(&cfg, fk, parts, np, sc);
    if (e != cudaSuccess) return fail(HPCCG_ECUDA, "p.Ap finisher launch: %s", cudaGetErrorString(e));
    return check_launch(ctx);
}

template <class K>
int wave(hpccg_ctx *ctx, K kernel) {
    const void *key = reinterpret_cast<const void *>(kernel);
    auto it = ctx->occ.find(key);
    if (it != ctx->occ.end()) return it->second;
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kernel, kBlock, 0) != cudaSuccess || b < 1) {
        cudaGetLastError();
        b = 1;
    }
    const int w = b * ctx->num_sms;
    ctx->occ[key] = w;
    return w;
}

// --------------------------------------------------------------- timing

cudaEvent_t pool_event(hpccg_problem *p) {
    if (p->ev_used == p->ev_pool.size()) {
        cudaEvent_t e;
        if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
        p->ev_pool.push_back(e);
    }
    return p->ev_pool[p->ev_used++];
}

struct PhaseTimer {  // records a begin/end event pair on `s` when timing is on
    hpccg_problem *p;
    cudaStream_t s;
    int phase;
    cudaEvent_t a = nullptr;
    PhaseTimer(hpccg_problem *p_, cudaStream_t s_, int ph, bool on) : p(p_), s(s_), phase(ph) {
        if (on) {
            a = pool_event(p);
            if (a) cudaEventRecord(a, s);
        }
    }
    ~PhaseTimer() {
        if (!a) return;
        cudaEvent_t b = pool_event(p);
        if (!b) return;
        cudaEventRecord(b, s);
        p->timed.push_back({phase, a, b});
    }
};

// ------------------------------------------------------- comm primitives

// Sum-allreduce (or max) of one scalar per slab: loc -> out, identical on all
// slabs / ranks.  Single: plain device copy is unnecessary (kernels write
// the global value directly), so this is only called for nslabs/nranks > 1.
int allreduce_scalar(hpccg_ctx *ctx, double *const *h_src, double *const *h_dst,
                     double *const *d_src, double *const *d_dst, bool is_max, int count = 1) {
    if (ctx->mode == MODE_LOOPBACK) {
        slab_allreduce_kernel<<<1, 32, 0, ctx->stream>>>(d_src, d_dst, ctx->nslabs, is_max, count);
        return check_launch(ctx);
    }
#ifdef HPCCG_WITH_NCCL
    if (ctx->mode == MODE_NCCL) {
        NC(ctx, ncclAllReduce(h_src[0], h_dst[0], count, ncclDouble, is_max ? ncclMax : ncclSum,
                              ctx->comm, ctx->stream));
        return HPCCG_OK;
    }
#endif
    (void)h_src;
    (void)h_dst;
    return fail(HPCCG_ENOTSUP, "allreduce: no communicator (peer-only contexts reduce per problem)");
}

// a.2 halo exchange of a local-with-halo vector per slab (bases xs[s]):
// first owned plane -> rank-1's upper halo, last owned plane -> rank+1's
// lower halo; the halo beyond the global z boundary is zero-filled.
// `on` = the stream the exchange runs on.
int exchange(hpccg_problem *p, double *const *xs, cudaStream_t on) {
    hpccg_ctx *ctx = p->ctx;
    const Slab &s0 = p->slabs[0];
    const int64_t n = s0.n, plane = s0.plane;
    const size_t pb = (size_t)plane * sizeof(double);
    if (ctx->mode == MODE_SINGLE) {
        CU(cudaMemsetAsync(xs[0], 0, pb, on));
        CU(cudaMemsetAsync(xs[0] + plane + n, 0, pb, on));
        return HPCCG_OK;
    }
    if (ctx->mode == MODE_LOOPBACK) {
        const int P = ctx->nslabs;
        for (int r = 0; r < P; ++r) {
            if (r > 0)  // my first owned plane -> (r-1)'s upper halo
                CU(cudaMemcpyAsync(xs[r - 1] + plane + n, xs[r] + plane, pb,
                                   cudaMemcpyDeviceToDevice, on));
            else
                CU(cudaMemsetAsync(xs[r], 0, pb, on));
            if (r < P - 1)  // my last owned plane -> (r+1)'s lower halo
                CU(cudaMemcpyAsync(xs[r + 1], xs[r] + n, pb, cudaMemcpyDeviceToDevice, on));
            else
                CU(cudaMemsetAsync(xs[r] + plane + n, 0, pb, on));
        }
        return HPCCG_OK;
    }
    if (ctx->mode == MODE_PEER)
        return fail(HPCCG_ENOTSUP, "peer-only context: no halo transport for caller-owned vectors");
#ifdef HPCCG_WITH_NCCL
    const int r = ctx->rank, P = ctx->nranks;
    double *x = xs[0];
    if (r == 0) CU(cudaMemsetAsync(x, 0, pb, on));
    if (r == P - 1) CU(cudaMemsetAsync(x + plane + n, 0, pb, on));
    NC(ctx, ncclGroupStart());
    if (r > 0) {
        NC(ctx, ncclSend(x + plane, plane, ncclDouble, r - 1, ctx->comm, on));
        NC(ctx, ncclRecv(x, plane, ncclDouble, r - 1, ctx->comm, on));
    }
    if (r < P - 1) {
        NC(ctx, ncclSend(x + n, plane, ncclDouble, r + 1, ctx->comm, on));
        NC(ctx, ncclRecv(x + plane + n, plane, ncclDouble, r + 1, ctx->comm, on));
    }
    NC(ctx, ncclGroupEnd());
    return HPCCG_OK;
#else
    return fail(HPCCG_ENOTSUP, "built without NCCL");
#endif
}

// HALO_PEER (multi-slab, opt_peer): the halo exchange as our own push /
// wait kernels over peer memory (kernels.cuh "peer-memory z-slab exchange").
bool peer_on(const hpccg_problem *p) { return p->opt_peer && p->ctx->mode != MODE_SINGLE; }
bool one_slab_per_process(const hpccg_ctx *ctx) { return ctx->mode == MODE_NCCL || ctx->mode == MODE_PEER; }

// push every hosted slab's boundary planes of x (local-with-halo bases xs)
int halo_push(hpccg_problem *p, double *const *xs, cudaStream_t on) {
    hpccg_ctx *ctx = p->ctx;
    const Slab &s0 = p->slabs[0];
    const int g = wave_grid(2 * s0.plane, wave(ctx, halo_push_kernel));
    for (size_t i = 0; i < p->slabs.size(); ++i) {
        halo_push_kernel<<<g, kBlock, 0, on>>>(p->slabs[i].ptab, xs[i], s0.n, s0.plane);
        CHECK(check_launch(ctx));
    }
    return HPCCG_OK;
}

int halo_wait(hpccg_problem *p, cudaStream_t on) {
    for (const Slab &s : p->slabs) {
        halo_wait_kernel<<<1, 32, 0, on>>>(s.ptab);
        CHECK(check_launch(p->ctx));
    }
    return HPCCG_OK;
}

// exchange of the internal gathered vector before an SpMV that does not
// overlap it (init): copies / NCCL, or push + wait
int halo_exchange(hpccg_problem *p, double *const *xs, cudaStream_t on) {
    if (!peer_on(p)) return exchange(p, xs, on);
    CHECK(halo_push(p, xs, on));
    return halo_wait(p, on);
}

// allreduce of `count` doubles per slab (src -> dst, identical on all slabs)
// over peer memory: posts of every hosted slab, then the collects (loopback
// hosts all slabs in one stream, so every post must precede every collect)
int peer_allreduce(hpccg_problem *p, double *const *src, double *const *dst, int count, bool is_max) {
    hpccg_ctx *ctx = p->ctx;
    const size_t P = p->slabs.size();
    if (P == 1) {
        peer_allreduce_kernel<<<1, 32, 0, ctx->stream>>>(p->slabs[0].ptab, src[0], dst[0], count, is_max, 1, 1);
        return check_launch(ctx);
    }
    for (size_t i = 0; i < P; ++i) {
        peer_allreduce_kernel<<<1, 32, 0, ctx->stream>>>(p->slabs[i].ptab, src[i], dst[i], count, is_max, 1, 0);
        CHECK(check_launch(ctx));
    }
    for (size_t i = 0; i < P; ++i) {
        peer_allreduce_kernel<<<1, 32, 0, ctx->stream>>>(p->slabs[i].ptab, src[i], dst[i], count, is_max, 0, 1);
        CHECK(check_launch(ctx));
    }
    return HPCCG_OK;
}

// ------------------------------------------------------------- launchers
// `check`: kernels test the device `done` flag first (plain launches and the
// per-iteration graph, which may run past convergence).  The while-graph
// never does, so its kernels skip that dependent load.

SpmvArgs spmv_args(const Slab &s, const double *x, double *y) {
    SpmvArgs a{};
    a.trace = s.trace_on ? s.trace : nullptr;
    a.trace_max = s.trace_max;
    a.stride = s.n;
    a.plane = s.plane;
    a.val = s.val;
    a.col = s.col;
    a.x = x;
    a.y = y;
    a.sc = s.sc;
    a.red = s.red;
    a.early_trigger = s.early_trigger;
    a.nx = s.nx;
    a.dia = s.dia;
    return a;
}

// kMinB of the SpMV (register budget): tuned on B200, see DESIGN.md sec. 7.
constexpr int kSpmvMinBDefault = 4;

template <int kDots, bool kCheck>
int launch_spmv_t(hpccg_ctx *ctx, int minb, const SpmvArgs &a, unsigned blocks, cudaStream_t st,
                  bool pdl) {
    switch (minb) {
        case 1: launch_k(pdl, spmv27_kernel<kDots, kCheck, 1>, dim3(blocks), st, a); break;
        case 3: launch_k(pdl, spmv27_kernel<kDots, kCheck, 3>, dim3(blocks), st, a); break;
        case 4: launch_k(pdl, spmv27_kernel<kDots, kCheck, 4>, dim3(blocks), st, a); break;
        default: launch_k(pdl, spmv27_kernel<kDots, kCheck, 2>, dim3(blocks), st, a); break;
    }
    return check_launch(ctx);
}

// Rows per thread of the SpMV for these ranges: 2 (spmv27x2_kernel) when the
// 16-B / 8-B slot loads are aligned (even n, even range starts, 16-B y).
int spmv_rows_per_thread(int opt_rows, const SpmvArgs &a, int64_t r0, int64_t r1) {
    if (opt_rows == 1) return 1;
    const bool ok = (a.stride % 2 == 0) && (r0 % 2 == 0) && (r1 % 2 == 0) && aligned16(a.y) &&
                    aligned16(a.val) && ((reinterpret_cast<uintptr_t>(a.col) & 7u) == 0);
    return ok ? 2 : 1;
}

int64_t spmv_blocks(int64_t len, int rows) { return cdiv(cdiv(len, rows), kBlock); }

template <int kDots>
int launch_spmv(hpccg_ctx *ctx, int minb, bool check, SpmvArgs a, int64_t r0, int64_t len0,
                int64_t r1, int64_t len1, cudaStream_t st, int rows = 1, bool pdl = false) {
    a.r0 = r0;
    a.len0 = len0;
    a.r1 = r1;
    a.len1 = len1;
    a.nb0 = spmv_blocks(len0, rows);
    a.nb01 = a.nb0 + spmv_blocks(len1, rows);
    const int64_t blocks = a.nb01 + spmv_blocks(a.len2, rows);  // len2: kFused only
    if (blocks == 0) return HPCCG_OK;
    if (blocks > 0x7fffffffLL) return fail(HPCCG_EINVAL, "SpMV grid too large");
    if (rows == 2) {
        if (a.dia) {
            if (check) launch_k(pdl, spmv27x2_kernel<kDots, true, false, true>, dim3((unsigned)blocks), st, a);
            else launch_k(pdl, spmv27x2_kernel<kDots, false, false, true>, dim3((unsigned)blocks), st, a);
        } else if (kDots == 1 && a.ring_n > 1) {  // p in a ring slot (ring-deferred x update)
            if (check) launch_k(pdl, spmv27x2_kernel<kDots, true, false, false, true>, dim3((unsigned)blocks), st, a);
            else launch_k(pdl, spmv27x2_kernel<kDots, false, false, false, true>, dim3((unsigned)blocks), st, a);
        } else if (check) {
            launch_k(pdl, spmv27x2_kernel<kDots, true>, dim3((unsigned)blocks), st, a);
        } else {
            launch_k(pdl, spmv27x2_kernel<kDots, false>, dim3((unsigned)blocks), st, a);
        }
        return check_launch(ctx);
    }
    if (minb <= 0) minb = kSpmvMinBDefault;
    return check ? launch_spmv_t<kDots, true>(ctx, minb, a, (unsigned)blocks, st, pdl)
                 : launch_spmv_t<kDots, false>(ctx, minb, a, (unsigned)blocks, st, pdl);
}

// y = A x for one slab over all rows (no dot).
int spmv_plain(hpccg_ctx *ctx, int minb, int opt_rows, const Slab &s, const double *x, double *y,
               cudaStream_t st) {
    SpmvArgs a = spmv_args(s, x, y);
    return launch_spmv<0>(ctx, minb, false, a, 0, s.n, 0, 0, st,
                              spmv_rows_per_thread(opt_rows, a, 0, 0));
}

// Blocks for `units` thread-units: the full grid, or `waves` resident waves.
template <class K>
int vec_grid(hpccg_ctx *ctx, K kernel, int64_t units, int waves, int64_t cap) {
    int64_t b = cdiv(std::max<int64_t>(units, 1), kBlock);
    if (waves > 0) b = std::min<int64_t>(b, (int64_t)waves * wave(ctx, kernel));
    return (int)std::max<int64_t>(1, std::min<int64_t>(b, cap));
}

template <bool kVec, bool kCheck, int kU>
int launch_pupdate_t(hpccg_ctx *ctx, int waves, const Slab &s, double *po, bool pdl) {
    auto k = cg_pupdate_kernel<kVec, kCheck, kU>;
    const int g = vec_grid(ctx, k, kVec ? cdiv(s.n, 2 * kU) : s.n, waves, 0x7fffffff);
    launch_k(pdl, k, dim3(g), ctx->stream, s.n, (const double *)s.r, po, (const CgScalars *)s.sc,
             s.trace_on ? s.trace : (TraceSlot *)nullptr, s.trace_max);
    return check_launch(ctx);
}

template <bool kVec, bool kCheck>
int launch_pupdate_u(hpccg_ctx *ctx, int waves, int unroll, const Slab &s, double *po, bool pdl) {
    switch (unroll) {
        case 1: return launch_pupdate_t<kVec, kCheck, 1>(ctx, waves, s, po, pdl);
        case 2: return launch_pupdate_t<kVec, kCheck, 2>(ctx, waves, s, po, pdl);
        default: return launch_pupdate_t<kVec, kCheck, 4>(ctx, waves, s, po, pdl);
    }
}

int launch_pupdate(hpccg_ctx *ctx, int waves, int unroll, const Slab &s, bool check, bool pdl) {
    double *po = s.p + s.plane;
    const bool vec = aligned16(s.r) && aligned16(po);
    if (vec)
        return check ? launch_pupdate_u<true, true>(ctx, waves, unroll, s, po, pdl)
                     : launch_pupdate_u<true, false>(ctx, waves, unroll, s, po, pdl);
    return check ? launch_pupdate_u<false, true>(ctx, waves, 1, s, po, pdl)
                 : launch_pupdate_u<false, false>(ctx, waves, 1, s, po, pdl);
}

template <bool kVec, bool kCheck, int kU>
int launch_update_t(hpccg_ctx *ctx, int waves, int64_t cap, const UpdArgs &a, bool pdl) {
    auto k = cg_update_kernel<kVec, kCheck, kU>;
    const int g = vec_grid(ctx, k, kVec ? cdiv(a.n, 2 * kU) : a.n, waves, cap);
    launch_k(pdl, k, dim3(g), ctx->stream, a);
    return check_launch(ctx);
}

template <bool kVec, bool kCheck>
int launch_update_u(hpccg_ctx *ctx, int waves, int unroll, int64_t cap, const UpdArgs &a, bool pdl) {
    switch (unroll) {
        case 1: return launch_update_t<kVec, kCheck, 1>(ctx, waves, cap, a, pdl);
        case 2: return launch_update_t<kVec, kCheck, 2>(ctx, waves, cap, a, pdl);
        default: return launch_update_t<kVec, kCheck, 4>(ctx, waves, cap, a, pdl);
    }
}

int launch_update(hpccg_ctx *ctx, int waves, int unroll, int64_t cap, const Slab &s, int single,
                  bool check, unsigned long long cond, bool pdl, int rows, int pap_cluster) {
    UpdArgs a{};
    a.n = s.n;
    a.x = s.x;
    a.r = s.r;
    a.p = s.p + s.plane;
    a.Ap = s.Ap;
    a.sc = s.sc;
    a.red = s.red;
    a.single = single;
    a.cond = cond;
    a.trace = s.trace_on ? s.trace : nullptr;
    a.trace_max = s.trace_max;
    if (single) {  // p.Ap partials of the single-slab SpMV (see cg_spmv_all)
        const unsigned np =
            (unsigned)spmv_blocks(s.n, spmv_rows_per_thread(rows, spmv_args(s, s.p, s.Ap), 0, 0));
        if (np <= kUpdSumMax) {  // every update block sums them
            a.pAp_parts = s.spmv_parts;
            a.n_parts = np;
        } else {  // the finisher writes sc->pAp, then the update reads it
            CHECK(launch_pap_finish(ctx, pap_cluster, s.spmv_parts, np, s.sc, pdl));
        }
    }
    const bool vec = aligned16(a.x) && aligned16(a.r) && aligned16(a.p) && aligned16(a.Ap);
    if (vec)
        return check ? launch_update_u<true, true>(ctx, waves, unroll, cap, a, pdl)
                     : launch_update_u<true, false>(ctx, waves, unroll, cap, a, pdl);
    return check ? launch_update_u<false, true>(ctx, waves, 1, cap, a, pdl)
                 : launch_update_u<false, false>(ctx, waves, 1, cap, a, pdl);
}

// Multi-slab SpMV around the halo exchange: the interior rows (planes
// 1..nz-2, no halo reads) overlap the exchange, the two boundary planes
// follow it.  NCCL: send/recv on the comm stream; HALO_PEER: our push kernel
// on the comm stream (NCCL ctx) or in stream order before the interiors
// (loopback), then a wait kernel before the boundaries; loopback copies: the
// exchange first.  slab_spmv(slab, interior) launches one part.
template <class F>
int spmv_overlapped(hpccg_problem *p, bool timing, double *const *xs, F slab_spmv) {
    hpccg_ctx *ctx = p->ctx;
    const bool peer = peer_on(p);
    if (one_slab_per_process(ctx)) {
        CU(cudaEventRecord(ctx->ev_fork, ctx->stream));
        CU(cudaStreamWaitEvent(ctx->comm_stream, ctx->ev_fork, 0));
        {
            PhaseTimer t(p, ctx->comm_stream, PH_EXCHANGE, timing);
            if (peer) CHECK(halo_push(p, xs, ctx->comm_stream));
            else CHECK(exchange(p, xs, ctx->comm_stream));
        }
        CU(cudaEventRecord(ctx->ev_join, ctx->comm_stream));
        PhaseTimer t(p, ctx->stream, PH_SPMV, timing);
        CHECK(slab_spmv(p->slabs[0], true));
        if (peer) CHECK(halo_wait(p, ctx->stream));
        CU(cudaStreamWaitEvent(ctx->stream, ctx->ev_join, 0));
        return slab_spmv(p->slabs[0], false);
    }
    {
        PhaseTimer t(p, ctx->stream, PH_EXCHANGE, timing);
        if (peer) CHECK(halo_push(p, xs, ctx->stream));
        else CHECK(exchange(p, xs, ctx->stream));
    }
    PhaseTimer t(p, ctx->stream, PH_SPMV, timing);
    if (peer) {
        for (const Slab &s : p->slabs) CHECK(slab_spmv(s, true));
        CHECK(halo_wait(p, ctx->stream));
        for (const Slab &s : p->slabs) CHECK(slab_spmv(s, false));
        return HPCCG_OK;
    }
    for (const Slab &s : p->slabs) {
        CHECK(slab_spmv(s, true));
        CHECK(slab_spmv(s, false));
    }
    return HPCCG_OK;
}

bool ff_path(const hpccg_problem *p);

// HPCCG_OPT_SERPENTINE in effect: auto = both bits once the CG vectors no
// longer fit in L2 (256^3: 1005.5 -> 999.0 us/iter; 128^3: no gain)
int serpentine(const hpccg_problem *p) {
    if (p->opt_serp >= 0) return p->opt_serp;
    return p->slabs[0].arena_bytes > ((size_t)126 << 20) ? 3 : 0;
}

// CG SpMV of every slab with the p.Ap epilogue.  Multi-slab: the rows that
// do not touch a halo plane (interior) run first, overlapped with the halo
// exchange on the comm stream (NCCL), then the two boundary planes.
// HPCCG_OPT_SPMV_SLICED: the single-slab CG SpMV (finisher-free loop) reads the
// chunk-sliced copy through TMA (spmv_sliced_kernel); auto = when the CG
// vectors exceed L2 (256^3 and up), where the copy's 324 B per row of extra HBM
// is cheap next to 180 GB
bool sliced_wanted(const hpccg_problem *p) {
    if (p->ctx->mode != MODE_SINGLE || p->opt_sliced == 0) return false;
    return p->opt_sliced == 1 || p->slabs[0].arena_bytes > ((size_t)126 << 20);
}

bool sliced_on(const hpccg_problem *p) {
    const Slab &s = p->slabs[0];
    return sliced_wanted(p) && s.sl && !s.dia && ff_path(p);
}

int alloc_zero(void **ptr, size_t bytes);

// allocate and fill the sliced copy (never during a graph capture: called at
// generate / set_option time)
int sliced_alloc(hpccg_problem *p) {
    Slab &s = p->slabs[0];
    if (s.sl || !sliced_wanted(p)) return HPCCG_OK;
    const int64_t nch = cdiv(s.n, kSlR);
    CHECK(alloc_zero((void **)&s.sl, (size_t)nch * kSlBytes));
    ell_to_sliced_kernel<<<(unsigned)cdiv(nch * kSlR, kBlock), kBlock, 0, p->ctx->stream>>>(
        s.n, s.plane, s.val, s.col, s.sl);
    CHECK(check_launch(p->ctx));
    CU(cudaStreamSynchronize(p->ctx->stream));
    return HPCCG_OK;
}

int sliced_grid(hpccg_ctx *ctx) {
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(spmv_sliced_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)(kSlStages * kSlBytes));
        cudaFuncSetAttribute(spmv_sliced_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)(kSlStages * kSlBytes));
        attr = true;
    }
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, spmv_sliced_kernel<false>, kSlR,
                                                      kSlStages * kSlBytes) != cudaSuccess || b < 1) {
        cudaGetLastError();
        b = 1;
    }
    return std::min(b, 2) * ctx->num_sms;
}

// HPCCG_OPT_SPMV_TRIPS: 512-row trips per block of the single-slab CG SpMV on
// the finisher-free loop (spmv27x2_trips_kernel), so the update blocks can sum
// the partials themselves (<= kUpdSumMax); 1: one trip (the finisher kernel
// runs when the partials exceed kUpdSumMax)
int spmv_trips(const hpccg_problem *p) {
    const Slab &s = p->slabs[0];
    if (p->ctx->mode != MODE_SINGLE || !ff_path(p) || s.dia || p->opt_spmv_trips == 1) return 1;
    if (spmv_rows_per_thread(p->opt_rows, spmv_args(s, s.p, s.Ap), 0, 0) != 2) return 1;
    const int64_t blocks = spmv_blocks(s.n, 2);
    if (p->opt_spmv_trips > 1) return p->opt_spmv_trips;
    return blocks > kUpdSumMax ? (int)cdiv(blocks, kUpdSumMax) : 1;
}

int defer_m(const hpccg_problem *p);
bool fuse_ps_on(hpccg_problem *p);

// HPCCG_OPT_SPMV_CLUSTER: the single-slab CG SpMV (finisher-free loop, 2 rows
// per thread) in clusters of kSpmvCl CTAs, one p.Ap partial per cluster; auto:
// when the per-CTA partials would exceed what the update blocks sum themselves
bool spmv_cl_on(const hpccg_problem *p) {
    if (p->ctx->mode != MODE_SINGLE || p->opt_spmv_cl == 0 || !ff_path(p)) return false;
    const Slab &s = p->slabs[0];
    if (s.dia || sliced_on(p) || spmv_trips(p) > 1 || fuse_ps_on(const_cast<hpccg_problem *>(p))) return false;
    if (spmv_rows_per_thread(p->opt_rows, spmv_args(s, s.p, s.Ap), 0, 0) != 2) return false;
    return p->opt_spmv_cl == 1 || spmv_blocks(s.n, 2) > (int64_t)kUpdSumMax;
}

int cg_spmv_all(hpccg_problem *p, bool timing, bool check) {
    hpccg_ctx *ctx = p->ctx;
    const int minb = p->opt_minb;
    if (ctx->mode == MODE_SINGLE) {
        const Slab &s = p->slabs[0];
        PhaseTimer t(p, ctx->stream, PH_SPMV, timing);
        SpmvArgs a = spmv_args(s, s.p, s.Ap);
        const int rows = spmv_rows_per_thread(p->opt_rows, a, 0, 0);
        a.single = 1;
        a.part_base = 0;
        a.total_blocks = (unsigned)spmv_blocks(s.n, rows);
        a.parts_only = s.spmv_parts;  // the update kernel finishes p.Ap
        a.rev = ff_path(p) && (serpentine(p) & 2);
        if (const int m = defer_m(p); m >= 2) {  // p_k in ring slot k % (m + 1)
            a.ring = s.pring;
            a.ring_stride = s.pring_stride;
            a.ring_n = m + 1;
        }
        if (sliced_on(p)) {
            a.r0 = 0;
            a.len0 = s.n;
            const unsigned g = (unsigned)sliced_grid(ctx);
            cudaLaunchConfig_t cfg{};
            cfg.gridDim = dim3(g);
            cfg.blockDim = dim3(kSlR);
            cfg.dynamicSmemBytes = kSlStages * kSlBytes;
            cfg.stream = ctx->stream;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            at[0].val.programmaticStreamSerializationAllowed = 1;
            cfg.attrs = p->opt_pdl ? at : nullptr;
            cfg.numAttrs = p->opt_pdl ? 1 : 0;
            const unsigned char *sl = s.sl;
            if (check) CU(cudaLaunchKernelEx(&cfg, spmv_sliced_kernel<true>, a, sl));
            else CU(cudaLaunchKernelEx(&cfg, spmv_sliced_kernel<false>, a, sl));
            return check_launch(ctx);
        }
        if (spmv_cl_on(p)) {
            a.r0 = 0;
            a.len0 = s.n;
            const int64_t nb = spmv_blocks(s.n, 2), g = cdiv(nb, kSpmvCl) * kSpmvCl;
            a.nb0 = g;
            a.total_blocks = (unsigned)g;
            cudaLaunchConfig_t cfg{};
            cfg.gridDim = dim3((unsigned)g);
            cfg.blockDim = dim3(kBlock);
            cfg.stream = ctx->stream;
            cudaLaunchAttribute at[2];
            int na = 0;
            at[na].id = cudaLaunchAttributeClusterDimension;
            at[na].val.clusterDim.x = kSpmvCl;
            at[na].val.clusterDim.y = 1;
            at[na++].val.clusterDim.z = 1;
            if (p->opt_pdl) {
                at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
                at[na++].val.programmaticStreamSerializationAllowed = 1;
            }
            cfg.attrs = at;
            cfg.numAttrs = na;
            if (a.ring_n > 1) {
                if (check) CU(cudaLaunchKernelEx(&cfg, spmv27x2_cl_kernel<true, true>, a));
                else CU(cudaLaunchKernelEx(&cfg, spmv27x2_cl_kernel<false, true>, a));
            } else {
                if (check) CU(cudaLaunchKernelEx(&cfg, spmv27x2_cl_kernel<true, false>, a));
                else CU(cudaLaunchKernelEx(&cfg, spmv27x2_cl_kernel<false, false>, a));
            }
            return check_launch(ctx);
        }
        const int trips = spmv_trips(p);
        if (trips > 1) {
            a.r0 = 0;
            a.len0 = s.n;
            a.trips = trips;
            const unsigned g = (unsigned)cdiv(spmv_blocks(s.n, 2), trips);
            if (check) launch_k(p->opt_pdl != 0, spmv27x2_trips_kernel<true>, dim3(g), ctx->stream, a);
            else launch_k(p->opt_pdl != 0, spmv27x2_trips_kernel<false>, dim3(g), ctx->stream, a);
            return check_launch(ctx);
        }
        return launch_spmv<1>(ctx, minb, check, a, 0, s.n, 0, 0, ctx->stream, rows,
                                 p->opt_pdl != 0);
    }
    const Slab &s0 = p->slabs[0];
    const int64_t n = s0.n, plane = s0.plane;
    // interior rows: planes 1..nz-2; boundary: plane 0 and plane nz-1
    const int64_t int_r0 = plane, int_len = std::max<int64_t>(n - 2 * plane, 0);
    const int64_t b0_len = std::min<int64_t>(plane, n);
    const int64_t b1_r0 = std::max<int64_t>(n - plane, plane), b1_len = n - b1_r0;
    const int rows = spmv_rows_per_thread(p->opt_rows, spmv_args(s0, s0.p, s0.Ap), int_r0, b1_r0);
    const unsigned nb_int = (unsigned)spmv_blocks(int_len, rows);
    const unsigned nb_bnd = (unsigned)(spmv_blocks(b0_len, rows) + spmv_blocks(b1_len, rows));
    std::vector<double *> xs(p->slabs.size());
    for (size_t i = 0; i < xs.size(); ++i) xs[i] = p->slabs[i].p;

    auto slab_spmv = [&](const Slab &s, bool interior) {
        SpmvArgs a = spmv_args(s, s.p, s.Ap);
        a.single = 0;
        a.total_blocks = nb_int + nb_bnd;
        if (interior) {
            a.part_base = 0;
            return launch_spmv<1>(ctx, minb, check, a, int_r0, int_len, 0, 0, ctx->stream, rows);
        }
        a.part_base = nb_int;
        return launch_spmv<1>(ctx, minb, check, a, 0, b0_len, b1_r0, b1_len, ctx->stream, rows);
    };
    return spmv_overlapped(p, timing, xs.data(), slab_spmv);
}

double **tab(hpccg_problem *p, int which) { return p->d_tab + (size_t)which * p->ctx->nslabs; }

// SpMV partial count of a single slab's CG SpMV (the update sums them).
unsigned single_spmv_parts(const hpccg_problem *p, const Slab &s) {
    if (sliced_on(p)) return (unsigned)sliced_grid(p->ctx);
    if (spmv_cl_on(p)) return (unsigned)cdiv(spmv_blocks(s.n, 2), kSpmvCl);
    const int trips = spmv_trips(p);
    if (trips > 1) return (unsigned)cdiv(spmv_blocks(s.n, 2), trips);
    return (unsigned)spmv_blocks(s.n, spmv_rows_per_thread(p->opt_rows, spmv_args(s, s.p, s.Ap), 0, 0));
}

int allreduce_cg(hpccg_problem *p, bool rr, bool timing) {
    hpccg_ctx *ctx = p->ctx;
    if (ctx->mode == MODE_SINGLE) return HPCCG_OK;
    PhaseTimer t(p, ctx->stream, PH_ALLREDUCE, timing);
    const Slab &s = p->slabs[0];
    if (peer_on(p)) {
        std::vector<double *> src, dst;
        for (const Slab &sl : p->slabs) {
            src.push_back(rr ? &sl.sc->loc_rr : &sl.sc->loc_pAp);
            dst.push_back(rr ? &sl.sc->rr_cur : &sl.sc->pAp);
        }
        return peer_allreduce(p, src.data(), dst.data(), 1, false);
    }
    double *hs[1] = {rr ? &s.sc->loc_rr : &s.sc->loc_pAp};
    double *hd[1] = {rr ? &s.sc->rr_cur : &s.sc->pAp};
    return allreduce_scalar(ctx, hs, hd, tab(p, rr ? 2 : 0), tab(p, rr ? 3 : 1), false);
}

// Single slab, HPCCG variant: the finisher-free loop (kernels.cuh
// cg_pupdate1 / cg_update1) when its vectors are 16-B aligned (always, for
// generated problems).
// HALO_PEER = 2: the halo exchange and both scalar allreduces of the HPCCG
// iteration fused into its three kernels (kernels.cuh "HALO_PEER = 2").
// It runs on the finisher-free loop (HPCCG_OPT_FINISHER_FREE, kernels
// cg_pupdate1 / spmv27x2<1, ., true> / cg_update1 with their peer hooks).
// Needs the 2-rows-per-thread SpMV and 16-B aligned vectors; else the
// HALO_PEER = 1 kernels run (same bits).
bool fused_on(const hpccg_problem *p) {
    if (p->opt_peer != 2 || !peer_on(p)) return false;
    if (p->opt_variant == 0 && !p->opt_ff) return false;  // HPCCG: on the finisher-free loop
    const Slab &s = p->slabs[0];
    if (!s.ptab || !aligned16(s.r) || !aligned16(s.p + s.plane) || !aligned16(s.x) || !aligned16(s.Ap) ||
        !aligned16(s.sv))
        return false;
    const int64_t b1_r0 = std::max<int64_t>(s.n - s.plane, s.plane);
    return spmv_rows_per_thread(p->opt_rows, spmv_args(s, s.p, s.Ap), s.plane, b1_r0) == 2;
}

// Blocks of a grid-stride vector grid (g blocks, 16-B unit i handled by
// thread i mod (g * kBlock)) that hold a unit of rows [0, plane) or
// [n - plane, n): the blocks that push a boundary plane.
// unit = 2: thread t holds the double2 units u == t (mod nth) (and thread 0
// the odd last row); unit = 1: the rows i == t (mod nth) (the ring-deferred p
// update's flush pass)
unsigned push_blocks(int64_t n, int64_t plane, int g, bool has_lo, bool has_hi, int unit = 2) {
    const int64_t nth = (int64_t)g * kBlock, nv = unit == 2 ? n >> 1 : n;
    std::vector<char> mark((size_t)g, 0);
    auto units = [&](int64_t u0, int64_t u1) {  // units [u0, u1)
        if (u1 <= u0) return;
        if (u1 - u0 >= nth) {
            std::fill(mark.begin(), mark.end(), 1);
            return;
        }
        for (int64_t t = u0 % nth, m = 0; m < u1 - u0;) {  // thread ranges, wrapping at nth
            const int64_t len = std::min(u1 - u0 - m, nth - t);
            for (int64_t b = t / kBlock; b <= (t + len - 1) / kBlock; ++b) mark[(size_t)b] = 1;
            m += len;
            t = 0;
        }
    };
    if (has_lo) units(0, std::min<int64_t>(cdiv(plane, unit), nv));  // units holding a row < plane
    if (has_hi) units(std::max<int64_t>((n - plane) / unit, 0), nv); // ... a row >= n - plane
    if (unit == 2 && (n & 1) && (has_hi || (has_lo && n - 1 < plane))) mark[0] = 1;  // thread 0: row n - 1
    return (unsigned)std::count(mark.begin(), mark.end(), 1);
}

// one launch per slab: interior row blocks, then plane 0, then plane nz-1
// (the same blocks and partial slots as HALO_PEER = 1's two launches)
template <int kDots = 1>
int launch_spmv_fused(hpccg_problem *p, const Slab &s, bool check, unsigned *nparts, int sr_q = 0) {
    const int64_t n = s.n, plane = s.plane;
    SpmvArgs a = spmv_args(s, s.p, s.Ap);
    a.single = 0;
    a.fpeer = s.ptab;
    a.r0 = plane;
    a.len0 = std::max<int64_t>(n - 2 * plane, 0);
    a.r1 = 0;
    a.len1 = std::min<int64_t>(plane, n);
    a.r2 = std::max<int64_t>(n - plane, plane);
    a.len2 = n - a.r2;
    a.nb0 = spmv_blocks(a.len0, 2);
    a.nb01 = a.nb0 + spmv_blocks(a.len1, 2);
    const int64_t blocks = a.nb01 + spmv_blocks(a.len2, 2);
    a.part_base = 0;
    a.total_blocks = (unsigned)blocks;
    a.parts_only = s.spmv_parts;  // the finisher-free update sums them
    *nparts = (unsigned)blocks;
    const bool pdl = p->opt_pdl != 0;
    a.sr_q = sr_q;
    if (kDots == 1) {
        if (const int m = defer_m(p); m >= 2) {  // p_k in ring slot k % (m + 1)
            a.ring = s.pring;
            a.ring_stride = s.pring_stride;
            a.ring_n = m + 1;
        }
    }
    if (kDots == 2) a.trace = nullptr;
    if (a.dia) {
        if (check) launch_k(pdl, spmv27x2_kernel<kDots, true, true, true>, dim3((unsigned)blocks), p->ctx->stream, a);
        else launch_k(pdl, spmv27x2_kernel<kDots, false, true, true>, dim3((unsigned)blocks), p->ctx->stream, a);
    } else if (kDots == 1 && a.ring_n > 1) {  // p in a ring slot (ring-deferred x update)
        if (check)
            launch_k(pdl, spmv27x2_kernel<kDots, true, true, false, true>, dim3((unsigned)blocks), p->ctx->stream, a);
        else
            launch_k(pdl, spmv27x2_kernel<kDots, false, true, false, true>, dim3((unsigned)blocks), p->ctx->stream, a);
    } else if (check) {
        launch_k(pdl, spmv27x2_kernel<kDots, true, true>, dim3((unsigned)blocks), p->ctx->stream, a);
    } else {
        launch_k(pdl, spmv27x2_kernel<kDots, false, true>, dim3((unsigned)blocks), p->ctx->stream, a);
    }
    return check_launch(p->ctx);
}

// the finisher-free HPCCG loop: single slab, or z-slabs with HALO_PEER = 2
bool ff_path(const hpccg_problem *p) {
    if (!p->opt_ff || p->opt_variant != 0) return false;
    if (p->ctx->mode != MODE_SINGLE) return fused_on(p);
    const Slab &s = p->slabs[0];
    return aligned16(s.r) && aligned16(s.p + s.plane) && aligned16(s.x) && aligned16(s.Ap);
}

// the deferred x update (HPCCG_OPT_DEFER_X) rides on the finisher-free loop
// (auto: when the CG vectors exceed L2 -- measured 256^3 989 vs 1005 us/iter,
// 128^3, vectors L2-resident, 115.1 vs 114.7: the x traffic then costs nothing)
bool defer_x_on(const hpccg_problem *p) {
    const bool on = p->opt_defer_x < 0 ? p->slabs[0].arena_bytes > ((size_t)126 << 20) : p->opt_defer_x != 0;
    return on && ff_path(p);
}

bool fuse_ps_on(hpccg_problem *p);
bool sliced_on(const hpccg_problem *p);
int spmv_trips(const hpccg_problem *p);

// auto depth of the ring-deferred x update (CG vectors beyond L2, single slab):
// tools/ringbench.cu -- the saving levels off from m = 6 (21.8 -> 21.9 -> 22.5 us
// per iteration at m = 6 / 8 / 12 at 256^3)
constexpr int kRingAutoM = kRingMaxM;

// the deferral depth in effect: 0 off, 1 every iteration (cg_pupdate1_kernel),
// m >= 2 over the ring (single slab on the plain finisher-free path only)
int defer_m(const hpccg_problem *p) {
    if (!defer_x_on(p)) return 0;
    const int want = p->opt_defer_x < 0 ? kRingAutoM : p->opt_defer_x;
    if (want < 2) return 1;
    for (const Slab &s : p->slabs)
        if (s.pring_slots < want || s.dia) return 1;
    if (p->ctx->mode != MODE_SINGLE)  // z-slabs: the peer tables must address the neighbours' rings
        return p->peer_ring ? want : 1;
    if (fuse_ps_on(const_cast<hpccg_problem *>(p)) || spmv_trips(p) > 1) return 1;
    return want;
}

// ring slots for depth m (never during a graph capture: generate / set_option)
int ring_alloc(hpccg_problem *p, int m) {
    if (m < 2) return HPCCG_OK;
    for (Slab &s : p->slabs) {
        if (s.pring_slots >= m) continue;
        // the neighbours of a one-slab-per-process context mapped the old ring at the
        // peer exchange: stop addressing rings (z-slabs run m = 1) rather than push
        // into freed memory; loopback tables are rebuilt by the caller
        if (s.ptab && one_slab_per_process(p->ctx)) p->peer_ring = false;
        cudaFree(s.pring_alloc);
        s.pring_alloc = s.pring = nullptr;
        s.pring_slots = 0;
        const int64_t seg = cdiv(s.ncol + 2, 32) * 32;  // as the arena's p segment
        CHECK(alloc_zero((void **)&s.pring_alloc, sizeof(double) * (size_t)(seg * m)));
        s.pring = s.pring_alloc + (s.p - s.p_alloc);  // the same 16-B alignment shift as p
        s.pring_stride = seg;
        s.pring_slots = m;
    }
    return HPCCG_OK;
}

PRing ring_of(const Slab &s, int m, bool owned) {
    PRing g{};
    g.base = s.pring + (owned ? s.plane : 0);
    g.stride = s.pring_stride;
    g.m = m;
    return g;
}

// f2 (single-reduction CG): x deferred over a ring of its p vector (s.r, not
// gathered, so no SpMV or halo change) -- HPCCG_OPT_DEFER_X as for HPCCG's loop
// (auto 8 beyond L2; 0 / 1: every iteration); the 2-rows/thread update only
int sr_ring_m(const hpccg_problem *p) {
    if (p->opt_variant != 1 || p->opt_defer_x == 0 || p->opt_defer_x == 1) return 0;
    if (p->opt_defer_x < 0 && p->slabs[0].arena_bytes <= ((size_t)126 << 20)) return 0;
    const int m = p->opt_defer_x < 0 ? kRingAutoM : p->opt_defer_x;
    for (const Slab &s : p->slabs)
        if (s.pring_slots < m || !aligned16(s.x) || !aligned16(s.p + s.plane) || !aligned16(s.r) ||
            !aligned16(s.sv) || !aligned16(s.Ap))
            return 0;
    return m;
}

// end of a solve on the finisher-free loop with the deferred x update: the
// last iteration's x += alpha p (cg_xfix_kernel; ring: the pending ones,
// cg_xfix_ring_kernel), every slab
int enqueue_xfix(hpccg_problem *p) {
    hpccg_ctx *ctx = p->ctx;
    if (const int m = sr_ring_m(p); m >= 2) {  // f2: update k flushes up to k itself
        for (const Slab &s : p->slabs) {
            PRing g = ring_of(s, m, true);
            launch_k(false, cg_xfix_ring_kernel, dim3(wave_grid(s.n / 2 + 1, wave(ctx, cg_xfix_ring_kernel))),
                     ctx->stream, (int64_t)s.n, s.x, s.r, g, (const CgScalars *)s.sc, 0);
            CHECK(check_launch(ctx));
        }
        return HPCCG_OK;
    }
    if (!defer_x_on(p)) return HPCCG_OK;
    if (const int m = defer_m(p); m >= 2) {
        for (const Slab &s : p->slabs) {
            launch_k(false, cg_xfix_ring_kernel, dim3(wave_grid(s.n / 2 + 1, wave(ctx, cg_xfix_ring_kernel))),
                     ctx->stream, (int64_t)s.n, s.x, s.p + s.plane, ring_of(s, m, true), (const CgScalars *)s.sc, 1);
            CHECK(check_launch(ctx));
        }
        return HPCCG_OK;
    }
    for (const Slab &s : p->slabs) {
        launch_k(false, cg_xfix_kernel, dim3(wave_grid(s.n / 2 + 1, wave(ctx, cg_xfix_kernel))),
                 ctx->stream, (int64_t)s.n, s.x, (const double *)(s.p + s.plane), (const CgScalars *)s.sc);
        CHECK(check_launch(ctx));
    }
    return HPCCG_OK;
}

// HPCCG_OPT_FUSE_PSPMV: single slab on the finisher-free loop, 2 rows per
// thread, a 128-B-aligned chunk layout (a line of p never spans two chunks).
// The lead (chunks between a block's production and its SpMV) must exceed
// the gather reach (plane + nx + 1 rows); past that, more lead = more time
// for a chunk's release to land before anyone needs it.
int64_t ps_lead(const hpccg_problem *p) {
    const Slab &s = p->slabs[0];
    const int64_t reach = (s.plane + s.nx + 1) / kPsRows + 2;
    return std::max<int64_t>(p->opt_ps_lead > 0 ? p->opt_ps_lead : reach + 128, reach + 1);
}

bool fuse_ps_on(hpccg_problem *p) {
    if (p->opt_fuse_ps == 0 || p->ctx->mode != MODE_SINGLE || p->opt_variant != 0 || !ff_path(p)) return false;
    const Slab &s = p->slabs[0];
    if (s.dia || (s.n & 1) || (s.plane & 15) || ((uintptr_t)(s.p + s.plane) & 127)) return false;
    if (spmv_rows_per_thread(p->opt_rows, spmv_args(s, s.p, s.Ap), 0, 0) != 2) return false;
    if (p->opt_fuse_ps < 0 && s.arena_bytes <= ((size_t)126 << 20)) return false;  // auto: vectors > L2
    return s.ps_mem != nullptr;  // allocated when the option is set (never during a graph capture)
}

int alloc_zero(void **ptr, size_t bytes);

int ps_alloc(Slab &s) {
    if (s.ps_mem) return HPCCG_OK;
    const int64_t nch = cdiv(s.n, kPsRows);
    const size_t bytes = 256 + sizeof(unsigned long long) * (size_t)nch;
    CHECK(alloc_zero((void **)&s.ps_mem, bytes));
    s.ps_ticket = (unsigned *)s.ps_mem;
    s.ps_err = (int *)(s.ps_mem + 64);
    s.ps_flags = (unsigned long long *)(s.ps_mem + 256);
    return HPCCG_OK;
}

// rows [row0, row0 + nrows) that the prologue p update handles: the first
// `lead` chunk positions (the last chunks when the SpMV walks backwards)
void ps_prologue_rows(const hpccg_problem *p, int64_t *row0, int64_t *nrows) {
    const Slab &s = p->slabs[0];
    const int64_t nch = cdiv(s.n, kPsRows), lead = std::min<int64_t>(ps_lead(p), nch);
    const bool rev = (serpentine(p) >> 1) & 1;
    *row0 = rev ? (nch - lead) * kPsRows : 0;
    *nrows = rev ? s.n - *row0 : std::min<int64_t>(lead * kPsRows, s.n);
}

int launch_pspmv(hpccg_problem *p, const Slab &s, int q) {
    PsArgs a{};
    a.n = s.n;
    a.plane = s.plane;
    a.nchunks = cdiv(s.n, kPsRows);
    a.nx = s.nx;
    a.lead = (int)ps_lead(p);
    a.rev = (serpentine(p) >> 1) & 1;
    a.q = q;
    a.val = s.val;
    a.col = s.col;
    a.p = s.p;
    a.r = s.r;
    a.x = defer_x_on(p) ? s.x : nullptr;
    a.Ap = s.Ap;
    a.parts = s.spmv_parts;
    a.sc = s.sc;
    a.ticket = s.ps_ticket;
    a.flags = s.ps_flags;
    a.trace = s.trace_on ? s.trace : nullptr;
    a.trace_max = s.trace_max;
    a.err = s.ps_err;
    launch_k(p->opt_pdl != 0, cg_pspmv_kernel, dim3((unsigned)a.nchunks), p->ctx->stream, a);
    return check_launch(p->ctx);
}

template <int kU>
int enqueue_iteration_ff_u(hpccg_problem *p, bool timing, bool check, unsigned long long cond, int q) {
    hpccg_ctx *ctx = p->ctx;
    const bool pdl = p->opt_pdl != 0;
    const bool zs = ctx->mode != MODE_SINGLE;  // HALO_PEER = 2 on z-slabs (fused_on)
    const bool fuse = !zs && fuse_ps_on(p);
    auto upd = zs ? cg_update1_kernel<kU, true> : fuse ? cg_update1_kernel<kU, false, true>
                                                       : cg_update1_kernel<kU, false>;
    auto pup = zs ? cg_pupdate1_kernel<kU, true> : cg_pupdate1_kernel<kU, false>;
    const Slab &s0 = p->slabs[0];
    // the update's grid fixes the r.r partials and so the bits: size it as
    // the finisher path's update kernel is sized, so both paths agree bitwise
    const int ug = vec_grid(ctx, cg_update_kernel<true, false, kU>, cdiv(s0.n, 2 * kU),
                            p->opt_vec_waves, p->red_cap);
    const int pg = vec_grid(ctx, pup, cdiv(s0.n, 2 * kU), p->opt_vec_waves, 0x7fffffff);
    // loopback: every slab's post ahead of every slab's collect (one stream)
    const bool pre = zs && ctx->mode == MODE_LOOPBACK;
    auto post = [&](const Slab &s, const double *parts, unsigned n, int q) {
        launch_k(pdl, fused_post_kernel, dim3(1), ctx->stream, parts, n, (const double *)&s.sc->pAp,
                 (const PeerTab *)s.ptab, (const CgScalars *)s.sc, q);
        return check_launch(ctx);
    };
    if (fuse) {  // the prologue p update (first `lead` chunks), then p update + SpMV in one kernel
        {
            PhaseTimer t(p, ctx->stream, PH_PUPDATE, timing);
            int64_t row0, nrows;
            ps_prologue_rows(p, &row0, &nrows);
            Pupd1Args a{};
            a.post = 1;
            a.n = nrows;
            a.r = s0.r + row0;
            a.p = s0.p + s0.plane + row0;
            a.rr_parts = s0.red.partials;
            a.n_rr = (unsigned)ug;
            a.sc = s0.sc;
            a.q = q;
            a.trace = s0.trace_on ? s0.trace : nullptr;
            a.trace_max = s0.trace_max;
            a.x = defer_x_on(p) ? s0.x + row0 : nullptr;
            const int gp = vec_grid(ctx, pup, cdiv(nrows, 2 * kU), p->opt_vec_waves, 0x7fffffff);
            launch_k(pdl, pup, dim3(gp), ctx->stream, a);
            CHECK(check_launch(ctx));
        }
        PhaseTimer t(p, ctx->stream, PH_SPMV, timing);
        CHECK(launch_pspmv(p, s0, q));
    } else if (const int m = defer_m(p); m >= 2) {  // ring-deferred x update
        PhaseTimer t(p, ctx->stream, PH_PUPDATE, timing);
        if (pre)
            for (const Slab &s : p->slabs) CHECK(post(s, s.red.partials, (unsigned)ug, 0));
        auto rk = zs ? cg_pupdate_ring_kernel<kU, true> : cg_pupdate_ring_kernel<kU, false>;
        const int rg = vec_grid(ctx, rk, cdiv(s0.n, 2 * kU), p->opt_vec_waves, 0x7fffffff);
        for (const Slab &s : p->slabs) {
            PringArgs a{};
            a.n = s.n;
            a.r = s.r;
            a.p = s.p + s.plane;
            a.ring = ring_of(s, m, true);
            a.x = s.x;
            a.rr_parts = s.red.partials;
            a.n_rr = (unsigned)ug;
            a.sc = s.sc;
            a.q = q;
            a.trace = s.trace_on ? s.trace : nullptr;
            a.trace_max = s.trace_max;
            a.rev = serpentine(p) & 1;
            a.post = !pre;
            if (zs) {
                const bool lo = s.rank > 0, hi = s.rank < ctx->nranks - 1;
                a.t = s.ptab;
                a.plane = s.plane;
                a.n_push = push_blocks(s.n, s.plane, rg, lo, hi, 2);
                a.n_push1 = push_blocks(s.n, s.plane, rg, lo, hi, 1);
            }
            launch_k(pdl, rk, dim3(rg), ctx->stream, a);
            CHECK(check_launch(ctx));
        }
    } else {
        PhaseTimer t(p, ctx->stream, PH_PUPDATE, timing);
        if (pre)
            for (const Slab &s : p->slabs) CHECK(post(s, s.red.partials, (unsigned)ug, 0));
        for (size_t si = 0; si < p->slabs.size(); ++si) {
            const Slab &s = p->slabs[si];
            Pupd1Args a{};
            a.post = !pre;
            a.n = s.n;
            a.r = s.r;
            a.p = s.p + s.plane;
            a.rr_parts = s.red.partials;
            a.n_rr = (unsigned)ug;
            a.sc = s.sc;
            a.q = q;
            a.trace = s.trace_on ? s.trace : nullptr;
            a.trace_max = s.trace_max;
            a.rev = serpentine(p) & 1;
            a.x = defer_x_on(p) ? s.x : nullptr;
            if (zs) {
                a.t = s.ptab;
                a.plane = s.plane;
                const uint64_t key = ((uint64_t)pg << 16) | ((uint64_t)kU << 8) | 2u;
                auto &cache = p->fpush[si];
                if (cache.first != key)
                    cache = {key, push_blocks(s.n, s.plane, pg, s.rank > 0, s.rank < ctx->nranks - 1)};
                a.n_push = cache.second;
            }
            launch_k(pdl, pup, dim3(pg), ctx->stream, a);
            CHECK(check_launch(ctx));
        }
    }
    unsigned np = 0;
    if (fuse) {
        np = (unsigned)cdiv(s0.n, kPsRows);
    } else if (zs) {
        PhaseTimer t(p, ctx->stream, PH_SPMV, timing);
        for (const Slab &s : p->slabs) CHECK(launch_spmv_fused(p, s, check, &np));
    } else {
        CHECK(cg_spmv_all(p, timing, check));
        np = single_spmv_parts(p, s0);
    }
    PhaseTimer t(p, ctx->stream, PH_UPDATE, timing);
    if (pre) {
        if (np > kUpdSumMax)
            for (const Slab &s : p->slabs) {  // sc->pAp = the slab's sum, then post it
                CHECK(launch_pap_finish(ctx, p->opt_pap_cluster, s.spmv_parts, np, s.sc, pdl));
            }
        for (const Slab &s : p->slabs)
            CHECK(post(s, np <= kUpdSumMax ? s.spmv_parts : nullptr, np, 1));
    }
    for (size_t si = 0; si < p->slabs.size(); ++si) {
        const Slab &s = p->slabs[si];
        Upd1Args a{};
        a.post = !pre;
        a.n = s.n;
        a.x = s.x;
        a.r = s.r;
        a.p = s.p + s.plane;
        a.Ap = s.Ap;
        a.rr_parts = s.red.partials;
        a.sc = s.sc;
        a.q = q;
        a.cond = si == 0 ? cond : 0ull;
        a.trace = s.trace_on ? s.trace : nullptr;
        a.trace_max = s.trace_max;
        a.t = zs ? s.ptab : nullptr;
        a.defer_x = defer_x_on(p) ? 1 : 0;
        if (np <= kUpdSumMax) {
            a.pAp_parts = s.spmv_parts;
            a.n_parts = np;
        } else if (pre) {  // finished and posted below, ahead of every update
        } else {  // the finisher writes the slab's p.Ap into sc->pAp
            CHECK(launch_pap_finish(ctx, p->opt_pap_cluster, s.spmv_parts, np, s.sc, pdl));
        }
        launch_k(pdl, upd, dim3(ug), ctx->stream, a);
        CHECK(check_launch(ctx));
    }
    return HPCCG_OK;
}

int enqueue_iteration_ff(hpccg_problem *p, bool timing, bool check, unsigned long long cond, int q) {
    switch (p->opt_unroll) {
        case 1: return enqueue_iteration_ff_u<1>(p, timing, check, cond, q);
        case 2: return enqueue_iteration_ff_u<2>(p, timing, check, cond, q);
        default: return enqueue_iteration_ff_u<4>(p, timing, check, cond, q);
    }
}

// One CG iteration (a.6, a.2, a.3+a.4, a.5, a.8) for every slab.  `cond`:
// while-graph condition handle (0 outside the while-graph); k: the
// iteration's index (its parity drives the finisher-free loop's state).
int enqueue_iteration(hpccg_problem *p, bool timing, bool check, unsigned long long cond, int k) {
    if (ff_path(p)) return enqueue_iteration_ff(p, timing, check, cond, k & 1);
    hpccg_ctx *ctx = p->ctx;
    const int single = ctx->mode == MODE_SINGLE;
    // PDL only between back-to-back kernels (single slab; the multi-slab
    // iteration has copies / NCCL calls between its kernels)
    const bool pdl = single && p->opt_pdl;
    {
        PhaseTimer t(p, ctx->stream, PH_PUPDATE, timing);
        for (const Slab &s : p->slabs)
            CHECK(launch_pupdate(ctx, p->opt_vec_waves, p->opt_unroll, s, check, pdl));
    }
    CHECK(cg_spmv_all(p, timing, check));
    CHECK(allreduce_cg(p, false, timing));
    {
        PhaseTimer t(p, ctx->stream, PH_UPDATE, timing);
        // every slab computes the same (allreduced) decision; slab 0 drives the
        // while-graph condition
        for (size_t i = 0; i < p->slabs.size(); ++i)
            CHECK(launch_update(ctx, p->opt_vec_waves, p->opt_unroll, p->red_cap, p->slabs[i],
                                single, check, i == 0 ? cond : 0ull, pdl, p->opt_rows, p->opt_pap_cluster));
    }
    CHECK(allreduce_cg(p, true, timing));
    return HPCCG_OK;
}

// a.7: p = x; halo; Ap = A p; r = b - Ap; rtrans = r.r; normr; first check.
int enqueue_init(hpccg_problem *p, int max_iter, double tol, bool timing,
                 unsigned long long cond) {
    hpccg_ctx *ctx = p->ctx;
    const int single = ctx->mode == MODE_SINGLE;
    for (const Slab &s : p->slabs) {
        copy_kernel<<<wave_grid(s.n, wave(ctx, copy_kernel)), kBlock, 0, ctx->stream>>>(
            s.n, s.x, s.p + s.plane);
        CHECK(check_launch(ctx));
    }
    std::vector<double *> xs(p->slabs.size());
    for (size_t i = 0; i < xs.size(); ++i) xs[i] = p->slabs[i].p;
    {
        PhaseTimer t(p, ctx->stream, PH_EXCHANGE, timing);
        CHECK(halo_exchange(p, xs.data(), ctx->stream));
    }
    {
        PhaseTimer t(p, ctx->stream, PH_SPMV, timing);
        for (const Slab &s : p->slabs)
            CHECK(spmv_plain(ctx, p->opt_minb, p->opt_rows, s, s.p, s.Ap, ctx->stream));
    }
    {
        PhaseTimer t(p, ctx->stream, PH_UPDATE, timing);
        for (const Slab &s : p->slabs) {
            InitResArgs a{};
            a.n = s.n;
            a.b = s.b;
            a.Ap = s.Ap;
            a.r = s.r;
            a.sc = s.sc;
            a.red = s.red;
            a.single = single;
            cg_initres_kernel<<<wave_grid(s.n, wave(ctx, cg_initres_kernel)), kBlock, 0,
                                ctx->stream>>>(a);
            CHECK(check_launch(ctx));
        }
    }
    CHECK(allreduce_cg(p, true, timing));
    for (size_t i = 0; i < p->slabs.size(); ++i) {
        cg_initstate_kernel<<<1, 1, 0, ctx->stream>>>(p->slabs[i].sc, max_iter, tol,
                                                      i == 0 ? cond : 0ull);
        CHECK(check_launch(ctx));
    }
    return HPCCG_OK;
}

// ------------------------------------ f2: single-reduction CG orchestration
// Buffers (same arena as HPCCG's CG): the GATHERED vector is r here, so r
// lives in the halo buffer s.p; w = A r in s.Ap; p (not gathered) in s.r;
// the s = A p recurrence in s.sv; x in s.x.

// w = A r with the (gamma, delta) epilogue for every slab; multi-slab: halo
// exchange overlapped with the interior rows (NCCL), per-slab finisher, and
// ONE allreduce of the two values.  q: parity of the iteration (run flag).
int cg_sr_spmv_all(hpccg_problem *p, bool timing, bool check, int q) {
    hpccg_ctx *ctx = p->ctx;
    const int minb = p->opt_minb;
    const bool pdl = ctx->mode == MODE_SINGLE && p->opt_pdl;
    auto finish = [&](const Slab &s, unsigned np, double *out) {
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(1);
        cfg.blockDim = dim3(1024);
        cfg.stream = ctx->stream;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = pdl ? at : nullptr;
        cfg.numAttrs = pdl ? 1 : 0;
        CU(cudaLaunchKernelEx(&cfg, cg_sr_finish_kernel, (const double *)s.spmv_parts, np, out));
        return check_launch(ctx);
    };
    if (ctx->mode == MODE_SINGLE) {
        const Slab &s = p->slabs[0];
        PhaseTimer t(p, ctx->stream, PH_SPMV, timing);
        SpmvArgs a = spmv_args(s, s.p, s.Ap);
        a.trace = nullptr;
        const int rows = spmv_rows_per_thread(p->opt_rows, a, 0, 0);
        a.single = 1;
        a.part_base = 0;
        a.total_blocks = (unsigned)spmv_blocks(s.n, rows);
        a.parts_only = s.spmv_parts;
        a.sr_q = q;
        CHECK(launch_spmv<2>(ctx, minb, check, a, 0, s.n, 0, 0, ctx->stream, rows, pdl));
        // too many partials for every update block to sum: one finisher block
        if (a.total_blocks > kUpdSumMax) CHECK(finish(s, a.total_blocks, s.sc->gd));
        return HPCCG_OK;
    }
    const Slab &s0 = p->slabs[0];
    const int64_t n = s0.n, plane = s0.plane;
    const int64_t int_r0 = plane, int_len = std::max<int64_t>(n - 2 * plane, 0);
    const int64_t b0_len = std::min<int64_t>(plane, n);
    const int64_t b1_r0 = std::max<int64_t>(n - plane, plane), b1_len = n - b1_r0;
    const int rows = spmv_rows_per_thread(p->opt_rows, spmv_args(s0, s0.p, s0.Ap), int_r0, b1_r0);
    const unsigned nb_int = (unsigned)spmv_blocks(int_len, rows);
    const unsigned nb_bnd = (unsigned)(spmv_blocks(b0_len, rows) + spmv_blocks(b1_len, rows));
    std::vector<double *> xs(p->slabs.size());
    for (size_t i = 0; i < xs.size(); ++i) xs[i] = p->slabs[i].p;
    auto slab_spmv = [&](const Slab &s, bool interior) {
        SpmvArgs a = spmv_args(s, s.p, s.Ap);
        a.trace = nullptr;
        a.single = 0;
        a.total_blocks = nb_int + nb_bnd;
        a.parts_only = s.spmv_parts;
        a.sr_q = q;
        if (interior) {
            a.part_base = 0;
            return launch_spmv<2>(ctx, minb, check, a, int_r0, int_len, 0, 0, ctx->stream, rows);
        }
        a.part_base = nb_int;
        return launch_spmv<2>(ctx, minb, check, a, 0, b0_len, b1_r0, b1_len, ctx->stream, rows);
    };
    CHECK(spmv_overlapped(p, timing, xs.data(), slab_spmv));
    for (const Slab &s : p->slabs) CHECK(finish(s, nb_int + nb_bnd, s.sc->loc_gd));
    PhaseTimer t(p, ctx->stream, PH_ALLREDUCE, timing);
    if (peer_on(p)) {
        std::vector<double *> src, dst;
        for (const Slab &sl : p->slabs) {
            src.push_back(sl.sc->loc_gd);
            dst.push_back(sl.sc->gd);
        }
        return peer_allreduce(p, src.data(), dst.data(), 2, false);
    }
    double *hs[1] = {p->slabs[0].sc->loc_gd};
    double *hd[1] = {p->slabs[0].sc->gd};
    return allreduce_scalar(ctx, hs, hd, tab(p, 6), tab(p, 7), false, 2);
}

template <bool kVec, int kU>
int launch_sr_update_t(hpccg_ctx *ctx, int waves, const SrUpdArgs &a, bool pdl) {
    auto k = cg_sr_update_kernel<kVec, kU>;
    const int g = vec_grid(ctx, k, kVec ? cdiv(a.n, 2 * kU) : a.n, waves, 0x7fffffff);
    launch_k(pdl, k, dim3(g), ctx->stream, a);
    return check_launch(ctx);
}

int launch_sr_update(hpccg_problem *p, const Slab &s, int q, unsigned long long cond, bool pdl) {
    hpccg_ctx *ctx = p->ctx;
    SrUpdArgs a{};
    a.n = s.n;
    a.x = s.x;
    a.r = s.p + s.plane;
    a.p = s.r;
    a.s = s.sv;
    a.w = s.Ap;
    a.sc = s.sc;
    a.q = q;
    a.cond = cond;
    if (const int m = sr_ring_m(p); m >= 2) a.ring = ring_of(s, m, true);
    if (ctx->mode == MODE_SINGLE) {
        const unsigned np = single_spmv_parts(p, s);
        if (np <= kUpdSumMax) {
            a.parts = s.spmv_parts;
            a.n_parts = np;
        }
    }
    const int waves = p->opt_vec_waves;
    const bool vec = aligned16(a.x) && aligned16(a.r) && aligned16(a.p) && aligned16(a.s) &&
                     aligned16(a.w);
    if (!vec) return launch_sr_update_t<false, 1>(ctx, waves, a, pdl);
    switch (p->opt_unroll) {
        case 1: return launch_sr_update_t<true, 1>(ctx, waves, a, pdl);
        case 2: return launch_sr_update_t<true, 2>(ctx, waves, a, pdl);
        default: return launch_sr_update_t<true, 4>(ctx, waves, a, pdl);
    }
}

// f2 with HALO_PEER = 2 on z-slabs: the update collects (gamma, delta) from
// every rank's post (block 0 posts the slab's; loopback: fused_post2_kernel
// ahead of every update) and pushes the new r's boundary planes into the
// neighbours' halos; the SpMV's boundary blocks wait for them; one post of
// two values per iteration.
template <int kU>
int enqueue_iteration_sr_fused_u(hpccg_problem *p, bool timing, bool check, unsigned long long cond, int q) {
    hpccg_ctx *ctx = p->ctx;
    const bool pdl = p->opt_pdl != 0;
    const bool pre = ctx->mode == MODE_LOOPBACK;
    auto upd = cg_sr_update_kernel<true, kU, true>;
    const Slab &s0 = p->slabs[0];
    const int g = vec_grid(ctx, upd, cdiv(s0.n, 2 * kU), p->opt_vec_waves, 0x7fffffff);
    // the slab sums come from cg_sr_finish_kernel (sc->loc_gd) as on the
    // HALO_PEER 0 / 1 z-slab path, so all three modes give the same bits
    {
        PhaseTimer t(p, ctx->stream, PH_UPDATE, timing);
        if (pre)
            for (const Slab &s : p->slabs) {
                launch_k(pdl, fused_post2_kernel, dim3(1), ctx->stream, (const double *)nullptr, 0u,
                         (const double *)s.sc->loc_gd, (const PeerTab *)s.ptab, (const CgScalars *)s.sc, q);
                CHECK(check_launch(ctx));
            }
        for (size_t si = 0; si < p->slabs.size(); ++si) {
            const Slab &s = p->slabs[si];
            SrUpdArgs a{};
            a.n = s.n;
            a.x = s.x;
            a.r = s.p + s.plane;
            a.p = s.r;
            a.s = s.sv;
            a.w = s.Ap;
            a.sc = s.sc;
            a.q = q;
            a.cond = si == 0 ? cond : 0ull;
            a.t = s.ptab;
            a.plane = s.plane;
            a.post = !pre;
            const uint64_t key = ((uint64_t)g << 16) | ((uint64_t)kU << 8) | 3u;
            auto &cache = p->fpush[si];
            if (cache.first != key)
                cache = {key, push_blocks(s.n, s.plane, g, s.rank > 0, s.rank < ctx->nranks - 1)};
            a.n_push = cache.second;
            if (const int m = sr_ring_m(p); m >= 2) {
                a.ring = ring_of(s, m, true);
                a.n_push1 = push_blocks(s.n, s.plane, g, s.rank > 0, s.rank < ctx->nranks - 1, 1);
            }
            launch_k(pdl, upd, dim3(g), ctx->stream, a);
            CHECK(check_launch(ctx));
        }
    }
    PhaseTimer t(p, ctx->stream, PH_SPMV, timing);
    unsigned npo = 0;
    for (const Slab &s : p->slabs) CHECK(launch_spmv_fused<2>(p, s, check, &npo, q));
    for (const Slab &s : p->slabs) {  // the slab sums for the next update (its loc_gd)
        launch_kb(pdl, cg_sr_finish_kernel, dim3(1), dim3(1024), ctx->stream, (const double *)s.spmv_parts, npo,
                  s.sc->loc_gd);
        CHECK(check_launch(ctx));
    }
    return HPCCG_OK;
}

// One f2 iteration of parity q: the fused update, then w = A r + (gamma, delta).
int enqueue_iteration_sr(hpccg_problem *p, bool timing, bool check, unsigned long long cond, int q) {
    hpccg_ctx *ctx = p->ctx;
    if (fused_on(p)) switch (p->opt_unroll) {
            case 1: return enqueue_iteration_sr_fused_u<1>(p, timing, check, cond, q);
            case 2: return enqueue_iteration_sr_fused_u<2>(p, timing, check, cond, q);
            default: return enqueue_iteration_sr_fused_u<4>(p, timing, check, cond, q);
        }
    const bool pdl = ctx->mode == MODE_SINGLE && p->opt_pdl;
    {
        PhaseTimer t(p, ctx->stream, PH_UPDATE, timing);
        for (size_t i = 0; i < p->slabs.size(); ++i)
            CHECK(launch_sr_update(p, p->slabs[i], q, i == 0 ? cond : 0ull, pdl));
    }
    return cg_sr_spmv_all(p, timing, check, q);
}

// f2 init: r = b - A x (r in the halo buffer), w = A r, (gamma, delta), state.
int enqueue_init_sr(hpccg_problem *p, int max_iter, double tol, bool timing,
                    unsigned long long cond) {
    hpccg_ctx *ctx = p->ctx;
    const int single = ctx->mode == MODE_SINGLE;
    for (const Slab &s : p->slabs) {
        copy_kernel<<<wave_grid(s.n, wave(ctx, copy_kernel)), kBlock, 0, ctx->stream>>>(
            s.n, s.x, s.p + s.plane);
        CHECK(check_launch(ctx));
    }
    std::vector<double *> xs(p->slabs.size());
    for (size_t i = 0; i < xs.size(); ++i) xs[i] = p->slabs[i].p;
    {
        PhaseTimer t(p, ctx->stream, PH_EXCHANGE, timing);
        CHECK(halo_exchange(p, xs.data(), ctx->stream));
    }
    {
        PhaseTimer t(p, ctx->stream, PH_SPMV, timing);
        for (const Slab &s : p->slabs)
            CHECK(spmv_plain(ctx, p->opt_minb, p->opt_rows, s, s.p, s.Ap, ctx->stream));
    }
    {
        PhaseTimer t(p, ctx->stream, PH_UPDATE, timing);
        for (const Slab &s : p->slabs) {  // r = b - A x0 (its r.r goes unused)
            InitResArgs a{};
            a.n = s.n;
            a.b = s.b;
            a.Ap = s.Ap;
            a.r = s.p + s.plane;
            a.sc = s.sc;
            a.red = s.red;
            a.single = single;
            cg_initres_kernel<<<wave_grid(s.n, wave(ctx, cg_initres_kernel)), kBlock, 0,
                                ctx->stream>>>(a);
            CHECK(check_launch(ctx));
        }
    }
    // HALO_PEER: a push must not land before every neighbour has finished
    // reading the previous exchange (the SpMV of A x just above); an allreduce
    // is that barrier (every rank posts only after its SpMV) -- everywhere
    // else in the solve one already separates consecutive exchanges
    if (peer_on(p)) CHECK(allreduce_cg(p, true, timing));
    CHECK(cg_sr_spmv_all(p, timing, false, 0));
    for (size_t i = 0; i < p->slabs.size(); ++i) {
        const Slab &s = p->slabs[i];
        const double *parts = nullptr;
        unsigned np = 0;
        if (single && single_spmv_parts(p, s) <= kUpdSumMax) {
            parts = s.spmv_parts;
            np = single_spmv_parts(p, s);
        }
        cg_sr_initstate_kernel<<<1, kBlock, 0, ctx->stream>>>(parts, np, s.sc, max_iter, tol,
                                                             i == 0 ? cond : 0ull);
        CHECK(check_launch(ctx));
    }
    return HPCCG_OK;
}

// Iterations captured per WHILE-body / per-iteration graph: f2 needs an even
// count (each launch's iteration parity is baked into the captured node).
int body_iterations(const hpccg_problem *p, int u) {
    if (p->opt_variant == 0 && !ff_path(p)) return u;
    return std::max(2, (u + 1) & ~1);
}

int enqueue_iteration_any(hpccg_problem *p, bool timing, bool check, unsigned long long cond, int k) {
    if (p->opt_variant == 1) return enqueue_iteration_sr(p, timing, check, cond, k & 1);
    return enqueue_iteration(p, timing, check, cond, k);
}

int enqueue_init_any(hpccg_problem *p, int max_iter, double tol, bool timing, unsigned long long cond) {
    if (p->opt_variant == 1) return enqueue_init_sr(p, max_iter, tol, timing, cond);
    return enqueue_init(p, max_iter, tol, timing, cond);
}

// L2 residency of the CG vectors (r, x, Ap, p: ~32n B): when they fit in the
// persisting L2 set-aside (cudaDevAttrMaxPersistingL2CacheSize, 74.6 MB on
// B200: n <= ~2.3M rows), an access-policy window marks the arena
// "persisting" while the matrix stream is loaded evict_first, so the vector
// kernels and the x gathers run out of L2 (measured at 128^3: 123.5 vs 132
// us/iteration).  When they do not fit, a window would pin a fraction of one
// vector and shrink the L2 for everything else (measured at 256^3: 1382 vs
// 1038 us/iteration), so it is not applied.  Applied to the stream (and so
// to every kernel captured into a graph) only for the solve; the set-aside
// is released and the persisting lines reset afterwards.
struct L2Window {
    hpccg_problem *p;
    bool on = false;
    size_t kept = 0;
    L2Window(hpccg_problem *p_, bool want) : p(p_) {
        hpccg_ctx *ctx = p->ctx;
        const Slab &s = p->slabs[0];
        if (!want || !p->opt_l2 || ctx->max_persist_l2 <= 0 || ctx->max_window <= 0) return;
        if (s.arena_bytes > (size_t)ctx->max_persist_l2 || s.arena_bytes > (size_t)ctx->max_window)
            return;
        if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, s.arena_bytes) != cudaSuccess) {
            cudaGetLastError();
            return;
        }
        cudaStreamAttrValue v{};
        v.accessPolicyWindow.base_ptr = s.arena;
        v.accessPolicyWindow.num_bytes = s.arena_bytes;
        v.accessPolicyWindow.hitRatio = 1.0f;
        v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        if (cudaStreamSetAttribute(ctx->stream, cudaStreamAttributeAccessPolicyWindow, &v) !=
            cudaSuccess) {
            cudaGetLastError();
            cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, 0);
            return;
        }
        on = true;
        size_t got = 0;
        kept = (cudaDeviceGetLimit(&got, cudaLimitPersistingL2CacheSize) == cudaSuccess) ? got : 0;
    }
    // call after the solve's work has completed
    void release() {
        if (!on) return;
        on = false;
        cudaStreamAttrValue v{};
        v.accessPolicyWindow.num_bytes = 0;
        cudaStreamSetAttribute(p->ctx->stream, cudaStreamAttributeAccessPolicyWindow, &v);
        cudaCtxResetPersistingL2Cache();
        cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, 0);
        cudaGetLastError();
    }
    ~L2Window() { release(); }
};

// Shared-memory-resident solve: bytes per row (ELL slice + vectors) and the
// rows per CTA when the problem fits one cluster (0: it does not).
// (DIA-27 reading, HPCCG_OPT_SPMV_FORMAT 1: no column slice)
int64_t smem_bytes_per_row(bool sr, bool dia) {
    return kSlots * (int64_t)(sizeof(double) + (dia ? 0 : sizeof(int))) + (sr ? 6 : 5) * (int64_t)sizeof(double);
}

int64_t smem_rows(const hpccg_problem *p) {
    const hpccg_ctx *ctx = p->ctx;
    if (!p->opt_smem || ctx->smem_cluster <= 1 || ctx->mode != MODE_SINGLE) return 0;
    const int64_t R = cdiv(p->slabs[0].n, ctx->smem_cluster);
    const bool sr = p->opt_variant == 1;
    // DIA (format 1) drops the column slice only where the ELL slice does not fit:
    // on chip, forming the column from the value costs more than reading it (DESIGN 7.1)
    if (R * smem_bytes_per_row(sr, false) <= ctx->smem_bytes) return R;
    return p->slabs[0].dia && R * smem_bytes_per_row(sr, true) <= ctx->smem_bytes ? R : 0;
}

// on-chip solve: halo rows per side of the gathered vector's local copy in
// every CTA (the stencil's reach, plane + nx + 1), 0 when it does not fit
// (the gathers then read the owner CTAs' shared memory)
int64_t smem_halo(const hpccg_problem *p, int64_t R, int64_t bytes_per_row) {
    if (p->opt_smem_halo == 0) return 0;
    const Slab &s = p->slabs[0];
    const int64_t H = s.plane + s.nx + 1;
    return R * bytes_per_row + 2 * H * (int64_t)sizeof(double) <= p->ctx->smem_bytes ? H : 0;
}

// the on-chip solve keeps no column slice (DIA reading): format 1 and the ELL slice does not fit
bool smem_dia(const hpccg_problem *p, int64_t R) {
    return p->slabs[0].dia && R * smem_bytes_per_row(p->opt_variant == 1, false) > p->ctx->smem_bytes;
}

// The whole solve in one cooperative kernel (small single-slab problems).
int launch_persistent(hpccg_problem *p, int max_iter, double tol) {
    hpccg_ctx *ctx = p->ctx;
    const Slab &s = p->slabs[0];
    PersistArgs a{};
    a.n = s.n;
    a.stride = s.n;
    a.plane = s.plane;
    a.val = s.val;
    a.col = s.col;
    a.b = s.b;
    a.x = s.x;
    a.r = s.r;
    a.p = s.p;
    a.Ap = s.Ap;
    a.part_rr = s.red.partials;
    a.part_pAp = s.red.partials + p->red_cap / 2;
    a.bar = s.bar;
    a.sc = s.sc;
    a.max_iter = max_iter;
    a.tol = tol;
    // whole problem in one cluster's shared memory when it fits
    const bool sr = p->opt_variant == 1;
    {
        const int64_t R = smem_rows(p);
        const int64_t bytes_per_row = smem_bytes_per_row(sr, smem_dia(p, R));
        if (R > 0) {
            SmemArgs m{};
            m.n = s.n;
            m.stride = s.n;
            m.plane = s.plane;
            m.R = (int)R;
            m.nx = s.nx;
            m.dia = smem_dia(p, R) ? 1 : 0;
            m.val = s.val;
            m.col = s.col;
            m.b = s.b;
            m.x = s.x;
            m.sc = s.sc;
            m.max_iter = max_iter;
            m.tol = tol;
            const int64_t H = smem_halo(p, R, bytes_per_row);
            m.H = (int)H;
            const int64_t g = cdiv(s.n, R);
            cudaLaunchConfig_t cfg{};
            // auto: 512 threads when a CTA holds more than 256 rows (one trip)
            const int nt = p->opt_smem_threads ? p->opt_smem_threads : (R > kBlock ? 512 : kBlock);
            cfg.gridDim = dim3((unsigned)g);
            cfg.blockDim = dim3(nt);
            cfg.dynamicSmemBytes = (size_t)(R * bytes_per_row + 2 * H * (int64_t)sizeof(double));
            cfg.stream = ctx->stream;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = (unsigned)g;
            at[0].val.clusterDim.y = 1;
            at[0].val.clusterDim.z = 1;
            cfg.attrs = at;
            cfg.numAttrs = 1;
            auto pick = [&](auto k512, auto k256) { return nt == 512 ? k512 : k256; };
            void (*kern)(SmemArgs) = nullptr;
            if (H > 0) {
                if (m.dia) kern = sr ? pick(cg_smem_cluster_kernel<512, true, true, true>, cg_smem_cluster_kernel<kBlock, true, true, true>)
                                     : pick(cg_smem_cluster_kernel<512, false, true, true>, cg_smem_cluster_kernel<kBlock, false, true, true>);
                else kern = sr ? pick(cg_smem_cluster_kernel<512, true, false, true>, cg_smem_cluster_kernel<kBlock, true, false, true>)
                               : pick(cg_smem_cluster_kernel<512, false, false, true>, cg_smem_cluster_kernel<kBlock, false, false, true>);
            } else {
                if (m.dia) kern = sr ? pick(cg_smem_cluster_kernel<512, true, true>, cg_smem_cluster_kernel<kBlock, true, true>)
                                     : pick(cg_smem_cluster_kernel<512, false, true>, cg_smem_cluster_kernel<kBlock, false, true>);
                else kern = sr ? pick(cg_smem_cluster_kernel<512, true>, cg_smem_cluster_kernel<kBlock, true>)
                               : pick(cg_smem_cluster_kernel<512, false>, cg_smem_cluster_kernel<kBlock, false>);
            }
            CU(cudaLaunchKernelEx(&cfg, kern, m));
            p->last_persist_mode = 5;
            return check_launch(ctx);
        }
    }
    if (s.n <= p->opt_cluster_rows && ctx->max_cluster > 1) {
        // one cluster of up to 16 CTAs, hardware cluster barrier between phases
        const int64_t g = std::max<int64_t>(1, std::min<int64_t>(cdiv(s.n, kBlock), ctx->max_cluster));
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3((unsigned)g);
        cfg.blockDim = dim3(kBlock);
        cfg.stream = ctx->stream;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = (unsigned)g;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        CU(cudaLaunchKernelEx(&cfg, cg_persistent_kernel<true>, a));
        p->last_persist_mode = 4;
    } else {
        int64_t g = std::min<int64_t>(cdiv(s.n, kBlock), wave(ctx, cg_persistent_kernel<false>));
        g = std::max<int64_t>(1, std::min<int64_t>(g, p->red_cap / 2));
        void *args[] = {&a};
        CU(cudaLaunchCooperativeKernel((const void *)cg_persistent_kernel<false>, dim3((unsigned)g),
                                       dim3(kBlock), args, 0, ctx->stream));
        p->last_persist_mode = 3;
    }
    return check_launch(ctx);
}

int build_graph(hpccg_problem *p) {
    hpccg_ctx *ctx = p->ctx;
    if (p->graph) return HPCCG_OK;
    cudaGraph_t g = nullptr;
    const int64_t l0 = ctx->launches;
    CU(cudaStreamBeginCapture(ctx->stream, cudaStreamCaptureModeThreadLocal));
    int rc = HPCCG_OK;
    for (int k = 1; k <= body_iterations(p, 1) && rc == HPCCG_OK; ++k)
        rc = enqueue_iteration_any(p, false, true, 0ull, k);
    cudaError_t e = cudaStreamEndCapture(ctx->stream, &g);
    if (rc != HPCCG_OK) {
        if (g) cudaGraphDestroy(g);
        return rc;
    }
    if (e != cudaSuccess) return fail(HPCCG_ECUDA, "graph capture: %s", cudaGetErrorString(e));
    p->graph_kernels = ctx->launches - l0;
    ctx->launches = l0;  // captured, not launched
    e = cudaGraphInstantiate(&p->graph, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess) {
        p->graph = nullptr;
        return fail(HPCCG_ECUDA, "graph instantiate: %s", cudaGetErrorString(e));
    }
    return HPCCG_OK;
}

// The whole solve as ONE graph: init, then a conditional WHILE node whose
// body is one CG iteration; the update kernel's last block sets the condition
// (= !done) on the device, so no host round trip until the solve ends.
// (max_iter, tol) are baked into the init kernel: rebuilt when they change.
int build_while_graph(hpccg_problem *p, int max_iter, double tol) {
    hpccg_ctx *ctx = p->ctx;
    if (p->wgraph && p->wgraph_max_iter == max_iter && p->wgraph_tol == tol) return HPCCG_OK;
    if (p->wgraph) {
        cudaGraphExecDestroy(p->wgraph);
        p->wgraph = nullptr;
    }
    cudaGraph_t g = nullptr;
    CU(cudaGraphCreate(&g, 0));
    auto bail = [&](int rc) {
        cudaGraphDestroy(g);
        return rc;
    };
    cudaGraphConditionalHandle h;
    if (cudaGraphConditionalHandleCreate(&h, g, 0, 0) != cudaSuccess)
        return bail(fail(HPCCG_ECUDA, "cudaGraphConditionalHandleCreate: %s",
                         cudaGetErrorString(cudaGetLastError())));
    const int64_t l0 = ctx->launches;
    // init, captured into g
    if (cudaStreamBeginCaptureToGraph(ctx->stream, g, nullptr, nullptr, 0,
                                      cudaStreamCaptureModeThreadLocal) != cudaSuccess)
        return bail(fail(HPCCG_ECUDA, "begin capture (init): %s",
                         cudaGetErrorString(cudaGetLastError())));
    int rc = enqueue_init_any(p, max_iter, tol, false, (unsigned long long)h);
    cudaStreamCaptureStatus cs;
    const cudaGraphNode_t *deps = nullptr;
    size_t ndeps = 0;
    cudaGraph_t cg = nullptr;
    if (rc == HPCCG_OK &&
        cudaStreamGetCaptureInfo(ctx->stream, &cs, nullptr, &cg, &deps, &ndeps) != cudaSuccess)
        rc = fail(HPCCG_ECUDA, "capture info");
    std::vector<cudaGraphNode_t> tail(deps, deps + ndeps);
    cudaGraph_t gout = nullptr;
    cudaError_t e = cudaStreamEndCapture(ctx->stream, &gout);
    if (rc != HPCCG_OK) return bail(rc);
    if (e != cudaSuccess) return bail(fail(HPCCG_ECUDA, "end capture (init): %s", cudaGetErrorString(e)));
    const int64_t l1 = ctx->launches;
    // while node after the init tail
    cudaGraphNodeParams cp{};
    cp.type = cudaGraphNodeTypeConditional;
    cp.conditional.handle = h;
    cp.conditional.type = cudaGraphCondTypeWhile;
    cp.conditional.size = 1;
    cudaGraphNode_t wnode;
    e = cudaGraphAddNode(&wnode, g, tail.data(), tail.size(), &cp);
    if (e != cudaSuccess) return bail(fail(HPCCG_ECUDA, "add while node: %s", cudaGetErrorString(e)));
    cudaGraph_t body = cp.conditional.phGraph_out[0];
    if (cudaStreamBeginCaptureToGraph(ctx->stream, body, nullptr, nullptr, 0,
                                      cudaStreamCaptureModeThreadLocal) != cudaSuccess)
        return bail(fail(HPCCG_ECUDA, "begin capture (body): %s",
                         cudaGetErrorString(cudaGetLastError())));
    // U iterations per WHILE-body execution: the per-execution cost of the
    // conditional node (~8 us measured with the device trace at 128^3) is paid
    // once per U iterations; with U > 1 the kernels test the device `done`
    // flag, so iterations after convergence inside a body are no-ops.
    const int U = body_iterations(p, std::max(1, p->opt_while_unroll));
    for (int u = 0; u < U && rc == HPCCG_OK; ++u)
        rc = enqueue_iteration_any(p, false, U > 1, (unsigned long long)h, 1 + u);
    e = cudaStreamEndCapture(ctx->stream, &gout);
    if (rc != HPCCG_OK) return bail(rc);
    if (e != cudaSuccess) return bail(fail(HPCCG_ECUDA, "end capture (body): %s", cudaGetErrorString(e)));
    p->wgraph_init_kernels = l1 - l0;
    p->wgraph_body_kernels = (ctx->launches - l1) / U;
    if (defer_x_on(p) || sr_ring_m(p) >= 2) {  // after the WHILE node: the deferred x update's pending ones
        const int64_t l2 = ctx->launches;
        if (cudaStreamBeginCaptureToGraph(ctx->stream, g, &wnode, nullptr, 1,
                                          cudaStreamCaptureModeThreadLocal) != cudaSuccess)
            return bail(fail(HPCCG_ECUDA, "begin capture (tail): %s", cudaGetErrorString(cudaGetLastError())));
        rc = enqueue_xfix(p);
        e = cudaStreamEndCapture(ctx->stream, &gout);
        if (rc != HPCCG_OK) return bail(rc);
        if (e != cudaSuccess) return bail(fail(HPCCG_ECUDA, "end capture (tail): %s", cudaGetErrorString(e)));
        p->wgraph_init_kernels += ctx->launches - l2;
    }
    ctx->launches = l0;
    e = cudaGraphInstantiate(&p->wgraph, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess) {
        p->wgraph = nullptr;
        return fail(HPCCG_ECUDA, "while-graph instantiate: %s", cudaGetErrorString(e));
    }
    p->whandle = h;
    p->wgraph_max_iter = max_iter;
    p->wgraph_tol = tol;
    return HPCCG_OK;
}

int alloc_zero(void **ptr, size_t bytes) {
    if (bytes == 0) bytes = 16;
    cudaError_t e = cudaMalloc(ptr, bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(HPCCG_ENOMEM, "cudaMalloc(%zu) failed: %s", bytes, cudaGetErrorString(e));
    }
    // cudaMemset runs on the legacy default stream, which does NOT order with
    // the library's non-blocking stream: wait for it, or a following kernel
    // on our stream can race with (and be overwritten by) the zero fill.
    e = cudaMemset(*ptr, 0, bytes);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return fail(HPCCG_ECUDA, "cudaMemset: %s", cudaGetErrorString(e));
    return HPCCG_OK;
}

void free_slab(Slab &s) {
    cudaFree(s.val);
    cudaFree(s.col);
    cudaFree(s.b);
    cudaFree(s.xexact);
    cudaFree(s.arena);
    cudaFree(s.sc);
    cudaFree(s.red.partials);
    cudaFree(s.red.counter);
    cudaFree(s.bar);
    cudaFree(s.spmv_parts);
    cudaFree(s.sv);
    cudaFree(s.psync);
    cudaFree(s.ptab);
    cudaFree(s.trace);
    cudaFree(s.ps_mem);
    cudaFree(s.sl);
    cudaFree(s.pring_alloc);
    s = Slab{};
}

int ctx_common_init(hpccg_ctx *c, int device, void *stream) {
    c->device = device;
    if (const char *e = getenv("HPCCG_AXPY_UNROLL")) c->axpy_unroll = atoi(e) == 4 ? 4 : 2;  // tuning knobs
    if (const char *e = getenv("HPCCG_DOT_UNROLL")) c->dot_unroll = atoi(e) == 2 ? 2 : 4;
    CU(cudaSetDevice(device));
    CU(cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device));
    CU(cudaDeviceGetAttribute(&c->max_persist_l2, cudaDevAttrMaxPersistingL2CacheSize, device));
    CU(cudaDeviceGetAttribute(&c->max_window, cudaDevAttrMaxAccessPolicyWindowSize, device));
    {   // shared-memory-resident solve: largest dynamic smem and cluster size
        int optin = 0;
        CU(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, device));
        c->smem_bytes = optin - 1024;  // static smem of the kernel + slack
        c->smem_cluster = 0;
        bool attr_ok = true;
        for (const void *k : {(const void *)cg_smem_cluster_kernel<kBlock, false>,
                              (const void *)cg_smem_cluster_kernel<kBlock, true>,
                              (const void *)cg_smem_cluster_kernel<512, false>,
                              (const void *)cg_smem_cluster_kernel<512, true>,
                              (const void *)cg_smem_cluster_kernel<kBlock, false, true>,
                              (const void *)cg_smem_cluster_kernel<kBlock, true, true>,
                              (const void *)cg_smem_cluster_kernel<512, false, true>,
                              (const void *)cg_smem_cluster_kernel<512, true, true>,
                              (const void *)cg_smem_cluster_kernel<kBlock, false, false, true>,
                              (const void *)cg_smem_cluster_kernel<kBlock, true, false, true>,
                              (const void *)cg_smem_cluster_kernel<512, false, false, true>,
                              (const void *)cg_smem_cluster_kernel<512, true, false, true>,
                              (const void *)cg_smem_cluster_kernel<kBlock, false, true, true>,
                              (const void *)cg_smem_cluster_kernel<kBlock, true, true, true>,
                              (const void *)cg_smem_cluster_kernel<512, false, true, true>,
                              (const void *)cg_smem_cluster_kernel<512, true, true, true>})
            attr_ok = attr_ok &&
                      cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           (int)c->smem_bytes) == cudaSuccess &&
                      cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) ==
                          cudaSuccess;
        if (attr_ok) {
            for (int sz : {16, 8}) {
                cudaLaunchConfig_t cfg{};
                cfg.gridDim = dim3(sz);
                cfg.blockDim = dim3(512);
                cfg.dynamicSmemBytes = (size_t)c->smem_bytes;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeClusterDimension;
                at[0].val.clusterDim.x = sz;
                at[0].val.clusterDim.y = 1;
                at[0].val.clusterDim.z = 1;
                cfg.attrs = at;
                cfg.numAttrs = 1;
                int ncl = 0;
                if (cudaOccupancyMaxActiveClusters(&ncl, cg_smem_cluster_kernel<512, true>, &cfg) ==
                        cudaSuccess &&
                    ncl > 0) {
                    c->smem_cluster = sz;
                    break;
                }
                cudaGetLastError();
            }
        }
        cudaGetLastError();
    }
    {   // largest cluster the persistent kernel can form (16 with the non-portable opt-in)
        int cc = 0;
        CU(cudaDeviceGetAttribute(&cc, cudaDevAttrClusterLaunch, device));
        c->max_cluster = 0;
        if (cc) {
            if (cudaFuncSetAttribute(cg_persistent_kernel<true>,
                                     cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess)
                cudaGetLastError();
            for (int sz : {16, 8, 4, 2}) {
                cudaLaunchConfig_t cfg{};
                cfg.gridDim = dim3(sz);
                cfg.blockDim = dim3(kBlock);
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeClusterDimension;
                at[0].val.clusterDim.x = sz;
                at[0].val.clusterDim.y = 1;
                at[0].val.clusterDim.z = 1;
                cfg.attrs = at;
                cfg.numAttrs = 1;
                int ncl = 0;
                if (cudaOccupancyMaxActiveClusters(&ncl, cg_persistent_kernel<true>, &cfg) == cudaSuccess &&
                    ncl > 0) {
                    c->max_cluster = sz;
                    break;
                }
                cudaGetLastError();
            }
        }
    }
    if (stream) {
        c->stream = (cudaStream_t)stream;
    } else {
        CU(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking));
        c->own_stream = true;
    }
    CU(cudaStreamCreateWithFlags(&c->comm_stream, cudaStreamNonBlocking));
    CU(cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
    CU(cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
    CHECK(alloc_zero((void **)&c->d_api, sizeof(double) * 2 * c->nslabs));
    CHECK(alloc_zero((void **)&c->d_api_src, sizeof(double *) * c->nslabs));
    CHECK(alloc_zero((void **)&c->d_api_dst, sizeof(double *) * c->nslabs));
    std::vector<double *> src(c->nslabs), dst(c->nslabs);
    for (int s = 0; s < c->nslabs; ++s) {
        src[s] = c->d_api + s;
        dst[s] = c->d_api + c->nslabs + s;
    }
    CU(cudaMemcpy(c->d_api_src, src.data(), sizeof(double *) * c->nslabs, cudaMemcpyHostToDevice));
    CU(cudaMemcpy(c->d_api_dst, dst.data(), sizeof(double *) * c->nslabs, cudaMemcpyHostToDevice));
    c->red_cap = 148 * 8 + 64;
    CHECK(alloc_zero((void **)&c->red.partials, sizeof(double) * c->red_cap));
    CHECK(alloc_zero((void **)&c->red.counter, sizeof(unsigned)));
    CU(cudaHostAlloc((void **)&c->h_pinned, 8 * sizeof(double), cudaHostAllocMapped));
    CU(cudaHostGetDevicePointer((void **)&c->d_mapped, c->h_pinned, 0));
    return HPCCG_OK;
}

// Reduce n-element vectors per slab with `launch(slab, x_s, y_s, out_s)` and
// allreduce the per-slab results; result on host.
// Single GPU: ONE kernel whose last block writes the result straight into
// mapped pinned host memory, then one stream sync -- no second kernel and no
// D2H copy (the two-kernel + copy DOT is what the paper blames for JACC's DOT
// overhead on GPUs).
template <class L>
int api_reduce(hpccg_ctx *ctx, bool is_max, double *result, L launch) {
    const bool single = ctx->mode == MODE_SINGLE;
    for (int s = 0; s < ctx->nslabs; ++s) {
        double *out = single ? ctx->d_mapped : ctx->d_api + s;
        CHECK(launch(s, out));
    }
    if (!single) {
        double *hs[1] = {ctx->d_api};
        double *hd[1] = {ctx->d_api + ctx->nslabs};
        CHECK(allreduce_scalar(ctx, hs, hd, ctx->d_api_src, ctx->d_api_dst, is_max));
        CU(cudaMemcpyAsync(ctx->h_pinned, ctx->d_api + ctx->nslabs, sizeof(double),
                           cudaMemcpyDeviceToHost, ctx->stream));
    }
    CU(cudaStreamSynchronize(ctx->stream));
    *result = *(volatile double *)ctx->h_pinned;
    return HPCCG_OK;
}

// HALO_PEER setup: every slab's PeerSync, then the peer tables.  Loopback:
// the neighbours' buffers are sibling slabs in this process.  One slab per
// process (NCCL or peer-only contexts): every rank exports its CG arena (which
// holds the halo'd vector) and its PeerSync as CUDA IPC handles (a "blob"),
// the blobs are all-gathered (over NCCL inside the library, or by the caller
// for peer-only contexts: hpccg_peer_export / hpccg_peer_attach) and the
// peers' buffers are mapped with cudaIpcOpenMemHandle (NVLink P2P between
// GPUs); the arena layout is identical on every rank, so a peer's vector sits
// at the same offset.
// the wait limit of every hosted slab's PeerSync (read by the spinning kernels)
int peer_set_timeout(hpccg_problem *p) {
    const unsigned long long ns = (unsigned long long)p->opt_peer_timeout_ms * 1000000ull;
    for (Slab &sl : p->slabs)
        if (sl.psync) CU(cudaMemcpy(&sl.psync->timeout_ns, &ns, sizeof ns, cudaMemcpyHostToDevice));
    return HPCCG_OK;
}

int peer_alloc(hpccg_problem *p) {
    if (p->ctx->nranks > kMaxPeers) return fail(HPCCG_ENOTSUP, "peer mode supports up to %d ranks", kMaxPeers);
    for (Slab &sl : p->slabs)
        if (!sl.psync) CHECK(alloc_zero((void **)&sl.psync, sizeof(PeerSync)));
    return peer_set_timeout(p);
}

// a timed-out wait -> HPCCG_ECUDA naming the rank, what it waited for and from whom
int peer_check_error(hpccg_problem *p, const char *op) {
    for (const Slab &sl : p->slabs) {
        int e[2] = {0, 0};  // error, error_peer (adjacent fields)
        CU(cudaMemcpy(e, &sl.psync->error, sizeof e, cudaMemcpyDeviceToHost));
        if (!e[0]) continue;
        static const char *what[] = {"?", "the halo plane of rank %d (lower neighbour)",
                                     "the halo plane of rank %d (upper neighbour)",
                                     "the allreduce post of rank %d", "the fused scalar post of rank %d"};
        char w[96];
        snprintf(w, sizeof w, what[e[0] >= 1 && e[0] <= 4 ? e[0] : 0], e[1]);
        return fail(HPCCG_ECUDA, "%s: peer-memory wait timed out after %lld ms on rank %d, waiting for %s",
                    op, (long long)p->opt_peer_timeout_ms, sl.rank, w);
    }
    return HPCCG_OK;
}


int peer_export(hpccg_problem *p, unsigned char *blob) {
    CHECK(peer_alloc(p));
    const Slab &s0 = p->slabs[0];
    memset(blob, 0, HPCCG_PEER_BLOB_BYTES);
    cudaIpcMemHandle_t h[2];
    CU(cudaIpcGetMemHandle(&h[0], s0.arena));
    CU(cudaIpcGetMemHandle(&h[1], s0.psync));
    memcpy(blob, h, sizeof h);
    if (s0.pring_alloc) {  // the p ring of the deferred x update (slot count in the last 4 bytes)
        cudaIpcMemHandle_t hr;
        CU(cudaIpcGetMemHandle(&hr, s0.pring_alloc));
        memcpy(blob + 2 * sizeof(cudaIpcMemHandle_t), &hr, sizeof hr);
        const int slots = s0.pring_slots;
        memcpy(blob + HPCCG_PEER_BLOB_BYTES - sizeof(int), &slots, sizeof slots);
    }
    return HPCCG_OK;
}

// sync[q] / pvec[q]: rank q's PeerSync and local-with-halo vector base (may
// be null for non-neighbours' vectors) -> device tables of the hosted slabs
// rvec[q]: rank q's p ring (halo base of slot 1; null: none / not a neighbour)
int peer_build_tables(hpccg_problem *p, const std::vector<PeerSync *> &sync,
                      const std::vector<double *> &pvec, const std::vector<double *> &rvec) {
    hpccg_ctx *ctx = p->ctx;
    const int P = ctx->nranks;
    const int64_t n = p->slabs[0].n, plane = p->slabs[0].plane;
    bool ring = true;
    for (size_t i = 0; i < p->slabs.size(); ++i) {
        Slab &sl = p->slabs[i];
        const int r = ctx->mode == MODE_LOOPBACK ? (int)i : ctx->rank;
        PeerTab t{};
        t.rank = r;
        t.nranks = P;
        t.mine = sl.psync;
        t.lo = r > 0 ? sync[r - 1] : nullptr;
        t.hi = r < P - 1 ? sync[r + 1] : nullptr;
        t.halo_to_lo = r > 0 ? pvec[r - 1] + plane + n : nullptr;
        t.halo_to_hi = r < P - 1 ? pvec[r + 1] : nullptr;
        t.ring_to_lo = r > 0 && rvec[r - 1] ? rvec[r - 1] + plane + n : nullptr;
        t.ring_to_hi = r < P - 1 ? rvec[r + 1] : nullptr;
        ring = ring && sl.pring && (r == 0 || t.ring_to_lo) && (r == P - 1 || t.ring_to_hi);
        for (int q = 0; q < P; ++q) t.all[q] = sync[q];
        if (!sl.ptab) CHECK(alloc_zero((void **)&sl.ptab, sizeof(PeerTab)));
        CU(cudaMemcpy(sl.ptab, &t, sizeof t, cudaMemcpyHostToDevice));
    }
    p->peer_ring = ring;
    return HPCCG_OK;
}

// blobs: nranks x HPCCG_PEER_BLOB_BYTES in rank order (one slab per process)
int peer_attach(hpccg_problem *p, const unsigned char *blobs) {
    hpccg_ctx *ctx = p->ctx;
    CHECK(peer_alloc(p));
    const int P = ctx->nranks, r = ctx->rank;
    const Slab &s0 = p->slabs[0];
    std::vector<PeerSync *> sync(P, nullptr);
    std::vector<double *> pvec(P, nullptr), rvec(P, nullptr);
    for (int q = 0; q < P; ++q) {
        if (q == r) {
            sync[q] = s0.psync;
            pvec[q] = s0.p;
            rvec[q] = s0.pring;
            continue;
        }
        cudaIpcMemHandle_t hq[2];
        memcpy(hq, blobs + (size_t)HPCCG_PEER_BLOB_BYTES * q, sizeof hq);
        void *ps = nullptr;
        CU(cudaIpcOpenMemHandle(&ps, hq[1], cudaIpcMemLazyEnablePeerAccess));
        p->ipc_opened.push_back(ps);
        sync[q] = (PeerSync *)ps;
        if (q == r - 1 || q == r + 1) {  // neighbours: their halo'd vector
            void *pa = nullptr;
            CU(cudaIpcOpenMemHandle(&pa, hq[0], cudaIpcMemLazyEnablePeerAccess));
            p->ipc_opened.push_back(pa);
            pvec[q] = (double *)pa + (s0.p - s0.arena);
            cudaIpcMemHandle_t hr, zero{};
            int slots = 0;
            memcpy(&hr, blobs + (size_t)HPCCG_PEER_BLOB_BYTES * q + 2 * sizeof(cudaIpcMemHandle_t), sizeof hr);
            memcpy(&slots, blobs + (size_t)HPCCG_PEER_BLOB_BYTES * (q + 1) - sizeof(int), sizeof slots);
            // the neighbour's ring, when both have one of the same depth (identical layouts)
            if (s0.pring && slots == s0.pring_slots && memcmp(&hr, &zero, sizeof hr) != 0) {
                void *pr = nullptr;
                CU(cudaIpcOpenMemHandle(&pr, hr, cudaIpcMemLazyEnablePeerAccess));
                p->ipc_opened.push_back(pr);
                rvec[q] = (double *)pr + (s0.pring - s0.pring_alloc);
            }
        }
    }
    return peer_build_tables(p, sync, pvec, rvec);
}

// HPCCG_OPT_HALO_PEER = 1 (collective): loopback and NCCL contexts build the
// tables themselves; peer-only contexts are attached by the caller.
int enable_peer(hpccg_problem *p) {
    hpccg_ctx *ctx = p->ctx;
    CHECK(peer_alloc(p));
    const int P = ctx->nranks;
    if (ctx->mode == MODE_LOOPBACK) {
        std::vector<PeerSync *> sync(P);
        std::vector<double *> pvec(P), rvec(P);
        for (int q = 0; q < P; ++q) {
            sync[q] = p->slabs[q].psync;
            pvec[q] = p->slabs[q].p;
            rvec[q] = p->slabs[q].pring;
        }
        return peer_build_tables(p, sync, pvec, rvec);
    }
    if (ctx->mode == MODE_NCCL) {
#ifdef HPCCG_WITH_NCCL
        const size_t B = HPCCG_PEER_BLOB_BYTES;
        std::vector<unsigned char> mine(B), all(B * P);
        CHECK(peer_export(p, mine.data()));
        unsigned char *d = nullptr;
        CU(cudaMalloc((void **)&d, B * (P + 1)));
        CU(cudaMemcpy(d, mine.data(), B, cudaMemcpyHostToDevice));
        ncclResult_t nr = ncclAllGather(d, d + B, B, ncclUint8, ctx->comm, ctx->stream);
        if (nr != ncclSuccess) {
            cudaFree(d);
            return nccl_fail(ctx, nr, "ncclAllGather(ipc handles)");
        }
        CU(cudaStreamSynchronize(ctx->stream));
        CU(cudaMemcpy(all.data(), d + B, B * P, cudaMemcpyDeviceToHost));
        cudaFree(d);
        return peer_attach(p, all.data());
#else
        return fail(HPCCG_ENOTSUP, "built without NCCL");
#endif
    }
    if (ctx->mode == MODE_PEER) return fail(HPCCG_EINVAL, "peer-only context: call hpccg_peer_attach");
    return HPCCG_OK;  // single GPU: nothing to exchange
}

}  // namespace

// ====================================================================== ABI

extern "C" {

const char *hpccg_strerror(int code) {
    switch (code) {
        case HPCCG_OK: return "HPCCG_OK";
        case HPCCG_EINVAL: return "HPCCG_EINVAL";
        case HPCCG_ENOMEM: return "HPCCG_ENOMEM";
        case HPCCG_ECUDA: return "HPCCG_ECUDA";
        case HPCCG_ENCCL: return "HPCCG_ENCCL";
        case HPCCG_ENOTSUP: return "HPCCG_ENOTSUP";
        default: return "HPCCG_E?";
    }
}

const char *hpccg_last_error(void) { return g_err.c_str(); }

const char *hpccg_version(void) {
#ifdef HPCCG_WITH_NCCL
    return "hpccg-b200 0.1 (sm_100a, nccl)";
#else
    return "hpccg-b200 0.1 (sm_100a)";
#endif
}

int hpccg_launch_count(const hpccg_ctx *ctx, int64_t *count) {
    if (!ctx || !count) return fail(HPCCG_EINVAL, "NULL argument");
    *count = ctx->launches;
    return HPCCG_OK;
}

int hpccg_unique_id(void *out) {
    if (!out) return fail(HPCCG_EINVAL, "NULL out");
#ifdef HPCCG_WITH_NCCL
    static_assert(sizeof(ncclUniqueId) == HPCCG_UNIQUE_ID_BYTES, "unique id size");
    ncclResult_t r = ncclGetUniqueId((ncclUniqueId *)out);
    if (r != ncclSuccess) return fail(HPCCG_ENCCL, "ncclGetUniqueId: %s", ncclGetErrorString(r));
    return HPCCG_OK;
#else
    return fail(HPCCG_ENOTSUP, "built without NCCL");
#endif
}

int hpccg_init(hpccg_ctx **out, int device, void *stream, int rank, int nranks,
               const void *unique_id) {
    if (!out || nranks < 1 || rank < 0 || rank >= nranks)
        return fail(HPCCG_EINVAL, "hpccg_init: bad rank/nranks");
    if (nranks > 1 && unique_id == nullptr)
        return fail(HPCCG_EINVAL, "hpccg_init: nranks > 1 needs the rank-0 unique_id");
    *out = nullptr;
    hpccg_ctx *c = new hpccg_ctx();
    c->rank = rank;
    c->nranks = nranks;
    c->nslabs = 1;
    // nranks == 1 with a unique_id: a 1-rank NCCL communicator running the
    // multi-GPU code path (halo split, NCCL allreduces, per-iteration graph)
    c->mode = unique_id == nullptr ? MODE_SINGLE : MODE_NCCL;
    int rc = ctx_common_init(c, device, stream);
    if (rc != HPCCG_OK) {
        hpccg_finalize(c);
        return rc;
    }
    if (c->mode == MODE_NCCL) {
#ifdef HPCCG_WITH_NCCL
        ncclUniqueId id;
        memcpy(&id, unique_id, sizeof id);
        ncclResult_t r = ncclCommInitRank(&c->comm, nranks, id, rank);
        if (r != ncclSuccess) {
            c->comm = nullptr;
            hpccg_finalize(c);
            return fail(HPCCG_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
        }
#else
        hpccg_finalize(c);
        return fail(HPCCG_ENOTSUP, "built without NCCL");
#endif
    }
    *out = c;
    return HPCCG_OK;
}

int hpccg_init_peer(hpccg_ctx **out, int device, void *stream, int rank, int nranks) {
    if (!out || nranks < 1 || rank < 0 || rank >= nranks || nranks > kMaxPeers)
        return fail(HPCCG_EINVAL, "hpccg_init_peer: bad rank/nranks");
    *out = nullptr;
    hpccg_ctx *c = new hpccg_ctx();
    c->rank = rank;
    c->nranks = nranks;
    c->nslabs = 1;
    c->mode = MODE_PEER;
    int rc = ctx_common_init(c, device, stream);
    if (rc != HPCCG_OK) {
        hpccg_finalize(c);
        return rc;
    }
    *out = c;
    return HPCCG_OK;
}

int hpccg_peer_export(hpccg_problem *p, void *blob) {
    if (!p || !blob) return fail(HPCCG_EINVAL, "NULL argument");
    if (!one_slab_per_process(p->ctx)) return fail(HPCCG_EINVAL, "peer export: one slab per process only");
    CU(cudaSetDevice(p->ctx->device));
    return peer_export(p, (unsigned char *)blob);
}

int hpccg_peer_attach(hpccg_problem *p, const void *blobs) {
    if (!p || !blobs) return fail(HPCCG_EINVAL, "NULL argument");
    if (!one_slab_per_process(p->ctx)) return fail(HPCCG_EINVAL, "peer attach: one slab per process only");
    if (p->slabs[0].ptab) return fail(HPCCG_EINVAL, "peer attach: already attached");
    CU(cudaSetDevice(p->ctx->device));
    CHECK(peer_attach(p, (const unsigned char *)blobs));
    if (p->graph) cudaGraphExecDestroy(p->graph);
    if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
    p->graph = p->wgraph = nullptr;
    p->opt_peer = 1;
    return HPCCG_OK;
}

int hpccg_init_loopback(hpccg_ctx **out, int device, void *stream, int nranks) {
    if (!out || nranks < 1) return fail(HPCCG_EINVAL, "hpccg_init_loopback: bad nranks");
    *out = nullptr;
    hpccg_ctx *c = new hpccg_ctx();
    c->rank = 0;
    c->nranks = nranks;
    c->nslabs = nranks;
    c->mode = nranks == 1 ? MODE_SINGLE : MODE_LOOPBACK;
    int rc = ctx_common_init(c, device, stream);
    if (rc != HPCCG_OK) {
        hpccg_finalize(c);
        return rc;
    }
    *out = c;
    return HPCCG_OK;
}

int hpccg_ctx_info(const hpccg_ctx *ctx, int *rank, int *nranks, int *nslabs) {
    if (!ctx) return fail(HPCCG_EINVAL, "NULL ctx");
    int r = ctx->rank, n = ctx->nranks;
#ifdef HPCCG_WITH_NCCL
    if (ctx->mode == MODE_NCCL && ctx->comm) {  // the communicator's own view
        ncclResult_t nr = ncclCommCount(ctx->comm, &n);
        if (nr == ncclSuccess) nr = ncclCommUserRank(ctx->comm, &r);
        if (nr != ncclSuccess) return fail(HPCCG_ENCCL, "ncclCommCount: %s", ncclGetErrorString(nr));
    }
#endif
    if (rank) *rank = r;
    if (nranks) *nranks = n;
    if (nslabs) *nslabs = ctx->nslabs;
    return HPCCG_OK;
}

void hpccg_finalize(hpccg_ctx *c) {
    if (!c) return;
    cudaSetDevice(c->device);
    if (c->stream) cudaStreamSynchronize(c->stream);
#ifdef HPCCG_WITH_NCCL
    if (c->comm) ncclCommDestroy(c->comm);
#endif
    cudaFree(c->d_api);
    cudaFree(c->d_api_src);
    cudaFree(c->d_api_dst);
    cudaFree(c->red.partials);
    cudaFree(c->red.counter);
    if (c->h_pinned) cudaFreeHost(c->h_pinned);
    if (c->ev_fork) cudaEventDestroy(c->ev_fork);
    if (c->ev_join) cudaEventDestroy(c->ev_join);
    if (c->comm_stream) cudaStreamDestroy(c->comm_stream);
    if (c->own_stream && c->stream) cudaStreamDestroy(c->stream);
    delete c;
}

int hpccg_generate(hpccg_ctx *ctx, int nx, int ny, int nz, hpccg_problem **out) {
    if (!ctx || !out) return fail(HPCCG_EINVAL, "NULL argument");
    if (nx < 1 || ny < 1 || nz < 1) return fail(HPCCG_EINVAL, "nx, ny, nz must be >= 1");
    const int64_t plane = (int64_t)nx * ny, n = plane * nz, ncol = n + 2 * plane;
    if (ncol >= 0x7fffffffLL) return fail(HPCCG_EINVAL, "local problem too large for int32 columns");
    if ((int64_t)nz * ctx->nranks >= 0x7fffffffLL) return fail(HPCCG_EINVAL, "nz * nranks too large");
    *out = nullptr;
    CU(cudaSetDevice(ctx->device));
    hpccg_problem *p = new hpccg_problem();
    p->ctx = ctx;
    p->nx = nx;
    p->ny = ny;
    p->nz = nz;
    p->slabs.resize(ctx->nslabs);
    p->fpush.assign((size_t)ctx->nslabs, {0ull, 0u});
    auto bail = [&](int rc) {
        hpccg_free(p);
        return rc;
    };
    for (int si = 0; si < ctx->nslabs; ++si) {
        Slab &s = p->slabs[si];
        s.rank = ctx->mode == MODE_LOOPBACK ? si : ctx->rank;
        s.n = n;
        s.plane = plane;
        s.ncol = ncol;
        s.nx = nx;
        int rc;
        if ((rc = alloc_zero((void **)&s.val, sizeof(double) * kSlots * n))) return bail(rc);
        if ((rc = alloc_zero((void **)&s.col, sizeof(int) * kSlots * n))) return bail(rc);
        if ((rc = alloc_zero((void **)&s.b, sizeof(double) * n))) return bail(rc);
        if ((rc = alloc_zero((void **)&s.xexact, sizeof(double) * n))) return bail(rc);
        // arena: [p (ncol + 2) | r | x | Ap], each segment 256-B aligned.
        // p: [lower halo | n owned | upper halo]; shifted by one element when
        // the plane is odd so the owned part is 16-B aligned (double2 loads).
        const int64_t seg_p = cdiv(ncol + 2, 32) * 32, seg_v = cdiv(n, 32) * 32;
        s.arena_bytes = sizeof(double) * (size_t)(seg_p + 3 * seg_v);
        if ((rc = alloc_zero((void **)&s.arena, s.arena_bytes))) return bail(rc);
        s.p_alloc = s.arena;
        s.p = s.p_alloc + ((plane & 1) ? 1 : 0);
        s.r = s.arena + seg_p;
        s.x = s.r + seg_v;
        s.Ap = s.x + seg_v;
        if ((rc = alloc_zero((void **)&s.sc, sizeof(CgScalars)))) return bail(rc);
        const int64_t parts = cdiv(n, kBlock) + 2 * cdiv(plane, kBlock) + 148 * 8 + 64;
        p->red_cap = parts;
        if ((rc = alloc_zero((void **)&s.red.partials, sizeof(double) * parts))) return bail(rc);
        if ((rc = alloc_zero((void **)&s.red.counter, sizeof(unsigned)))) return bail(rc);
        if ((rc = alloc_zero((void **)&s.bar, 64 * sizeof(unsigned)))) return bail(rc);
        if ((rc = alloc_zero((void **)&s.spmv_parts, sizeof(double) * 2 * parts))) return bail(rc);
        if ((rc = alloc_zero((void **)&s.sv, sizeof(double) * (size_t)(cdiv(n, 32) * 32)))) return bail(rc);

        GenArgs g{};
        g.nx = nx;
        g.ny = ny;
        g.nz = nz;
        g.rank = s.rank;
        g.nranks = ctx->nranks;
        g.n = n;
        g.plane = plane;
        g.val = s.val;
        g.col = s.col;
        g.b = s.b;
        g.x = s.x;
        g.xexact = s.xexact;
        g.nnz = &s.sc->nnz;
        const int64_t blocks = cdiv(n, kBlock);
        gen27_kernel<<<(unsigned)blocks, kBlock, 0, ctx->stream>>>(g);
        if ((rc = check_launch(ctx))) return bail(rc);
    }
    if (cudaStreamSynchronize(ctx->stream) != cudaSuccess)
        return bail(fail(HPCCG_ECUDA, "generate: %s", cudaGetErrorString(cudaGetLastError())));
    unsigned long long local = 0;
    for (Slab &s : p->slabs) {
        if (cudaMemcpy(&s.nnz, &s.sc->nnz, sizeof s.nnz, cudaMemcpyDeviceToHost) != cudaSuccess)
            return bail(fail(HPCCG_ECUDA, "generate: nnz readback"));
        local += s.nnz;
    }
    p->nnz_global = local;
    if (ctx->mode == MODE_PEER)  // no collective transport here: the closed form (pinned by the oracle)
        p->nnz_global = (unsigned long long)(3LL * nx - 2) * (unsigned long long)(3LL * ny - 2) *
                        (unsigned long long)(3LL * nz * ctx->nranks - 2);
#ifdef HPCCG_WITH_NCCL
    if (ctx->mode == MODE_NCCL) {
        unsigned long long *d = nullptr;
        int rc;
        if ((rc = alloc_zero((void **)&d, sizeof *d))) return bail(rc);
        cudaMemcpy(d, &local, sizeof local, cudaMemcpyHostToDevice);
        ncclResult_t r = ncclAllReduce(d, d, 1, ncclUint64, ncclSum, ctx->comm, ctx->stream);
        if (r != ncclSuccess) {
            cudaFree(d);
            return bail(nccl_fail(ctx, r, "ncclAllReduce(nnz)"));
        }
        cudaStreamSynchronize(ctx->stream);
        cudaMemcpy(&p->nnz_global, d, sizeof local, cudaMemcpyDeviceToHost);
        cudaFree(d);
    }
#endif
    // loopback allreduce pointer tables
    if (ctx->mode == MODE_LOOPBACK) {
        const int P = ctx->nslabs;
        int rc;
        if ((rc = alloc_zero((void **)&p->d_tab, sizeof(double *) * 8 * P))) return bail(rc);
        std::vector<double *> t(8 * P);
        for (int s = 0; s < P; ++s) {
            CgScalars *sc = p->slabs[s].sc;
            t[0 * P + s] = &sc->loc_pAp;
            t[1 * P + s] = &sc->pAp;
            t[2 * P + s] = &sc->loc_rr;
            t[3 * P + s] = &sc->rr_cur;
            t[4 * P + s] = &sc->red_loc;
            t[5 * P + s] = &sc->red_out;
            t[6 * P + s] = &sc->loc_gd[0];
            t[7 * P + s] = &sc->gd[0];
        }
        if (cudaMemcpy(p->d_tab, t.data(), sizeof(double *) * 8 * P, cudaMemcpyHostToDevice) !=
            cudaSuccess)
            return bail(fail(HPCCG_ECUDA, "generate: table upload"));
    }
    if (cudaMallocHost((void **)&p->h_done, 2 * sizeof(int)) != cudaSuccess)
        return bail(fail(HPCCG_ENOMEM, "pinned alloc"));
    if (cudaEventCreate(&p->ev_t0) != cudaSuccess || cudaEventCreate(&p->ev_t1) != cudaSuccess ||
        cudaEventCreateWithFlags(&p->ev_poll[0], cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&p->ev_poll[1], cudaEventDisableTiming) != cudaSuccess)
        return bail(fail(HPCCG_ECUDA, "event create"));
    if (ctx->mode == MODE_SINGLE) {  // the CG SpMV's chunk-sliced copy (auto: large problems)
        int rc = sliced_alloc(p);
        if (rc) return bail(rc);
    }
    // the p rings of the deferred x update (auto: CG vectors beyond L2), before any
    // peer exchange so the neighbours can address them.  Best effort: a problem that
    // fits without its ring still runs (x deferred by one iteration) when the m more
    // p-sized buffers do not fit
    if (p->slabs[0].arena_bytes > ((size_t)126 << 20) && ring_alloc(p, kRingAutoM) != HPCCG_OK) {
        for (Slab &s : p->slabs) {
            cudaFree(s.pring_alloc);
            s.pring_alloc = s.pring = nullptr;
            s.pring_slots = 0;
        }
        cudaGetLastError();
    }
    *out = p;
    return HPCCG_OK;
}

int hpccg_info(const hpccg_problem *p, int64_t *nrow_local, int64_t *ncol_local,
               int64_t *nnz_local, int64_t *nrow_global, int64_t *nnz_global) {
    if (!p) return fail(HPCCG_EINVAL, "NULL problem");
    const Slab &s = p->slabs[0];
    unsigned long long loc = 0;
    for (const Slab &q : p->slabs) loc += q.nnz;
    if (nrow_local) *nrow_local = s.n;
    if (ncol_local) *ncol_local = s.ncol;
    if (nnz_local) *nnz_local = (int64_t)loc;
    if (nrow_global) *nrow_global = s.n * p->ctx->nranks;
    if (nnz_global) *nnz_global = (int64_t)p->nnz_global;
    return HPCCG_OK;
}

static double *slab_vec(const Slab &s, int which) {
    switch (which) {
        case HPCCG_VEC_X: return s.x;
        case HPCCG_VEC_B: return s.b;
        case HPCCG_VEC_XEXACT: return s.xexact;
        default: return nullptr;
    }
}

int hpccg_vec(hpccg_problem *p, int which, double **dev_ptr) {
    if (!p || !dev_ptr) return fail(HPCCG_EINVAL, "NULL argument");
    if (p->slabs.size() > 1)
        return fail(HPCCG_ENOTSUP, "hpccg_vec: loopback slabs are separate allocations; "
                                   "use hpccg_get_vec / hpccg_set_vec");
    double *v = slab_vec(p->slabs[0], which);
    if (!v) return fail(HPCCG_EINVAL, "bad vector id %d", which);
    *dev_ptr = v;
    return HPCCG_OK;
}

int hpccg_set_vec(hpccg_problem *p, int which, const double *host_src) {
    if (!p || !host_src) return fail(HPCCG_EINVAL, "NULL argument");
    CU(cudaSetDevice(p->ctx->device));
    for (size_t i = 0; i < p->slabs.size(); ++i) {
        const Slab &s = p->slabs[i];
        double *v = slab_vec(s, which);
        if (!v) return fail(HPCCG_EINVAL, "bad vector id %d", which);
        CU(cudaMemcpyAsync(v, host_src + i * s.n, sizeof(double) * s.n, cudaMemcpyHostToDevice,
                           p->ctx->stream));
    }
    CU(cudaStreamSynchronize(p->ctx->stream));
    return HPCCG_OK;
}

int hpccg_get_vec(const hpccg_problem *p, int which, double *host_dst) {
    if (!p || !host_dst) return fail(HPCCG_EINVAL, "NULL argument");
    CU(cudaSetDevice(p->ctx->device));
    for (size_t i = 0; i < p->slabs.size(); ++i) {
        const Slab &s = p->slabs[i];
        double *v = slab_vec(s, which);
        if (!v) return fail(HPCCG_EINVAL, "bad vector id %d", which);
        CU(cudaMemcpyAsync(host_dst + i * s.n, v, sizeof(double) * s.n, cudaMemcpyDeviceToHost,
                           p->ctx->stream));
    }
    CU(cudaStreamSynchronize(p->ctx->stream));
    return HPCCG_OK;
}

int hpccg_copy_matrix(const hpccg_problem *p, int slab, double *val_host, int32_t *col_host) {
    if (!p || !val_host || !col_host) return fail(HPCCG_EINVAL, "NULL argument");
    if (slab < 0 || slab >= (int)p->slabs.size()) return fail(HPCCG_EINVAL, "bad slab");
    CU(cudaSetDevice(p->ctx->device));
    const Slab &s = p->slabs[slab];
    CU(cudaMemcpyAsync(val_host, s.val, sizeof(double) * kSlots * s.n, cudaMemcpyDeviceToHost,
                       p->ctx->stream));
    CU(cudaMemcpyAsync(col_host, s.col, sizeof(int) * kSlots * s.n, cudaMemcpyDeviceToHost,
                       p->ctx->stream));
    CU(cudaStreamSynchronize(p->ctx->stream));
    return HPCCG_OK;
}

int hpccg_set_option(hpccg_problem *p, int key, int64_t value) {
    if (!p) return fail(HPCCG_EINVAL, "NULL problem");
    // captured graphs bake in the launch configuration: rebuild on change
    cudaSetDevice(p->ctx->device);
    if (p->graph) cudaGraphExecDestroy(p->graph);
    if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
    p->graph = nullptr;
    p->wgraph = nullptr;
    p->while_failed = false;
    switch (key) {
        case HPCCG_OPT_GRAPH: p->opt_graph = value != 0; return HPCCG_OK;
        case HPCCG_OPT_POLL:
            if (value < 0) return fail(HPCCG_EINVAL, "poll must be >= 0");
            p->opt_poll = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_TIMING: p->opt_timing = value != 0; return HPCCG_OK;
        case HPCCG_OPT_SPMV_MINB:
            if (value < 0 || value > 4) return fail(HPCCG_EINVAL, "spmv minb must be 0..4");
            p->opt_minb = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_WHILE: p->opt_while = value != 0; return HPCCG_OK;
        case HPCCG_OPT_L2_PERSIST: p->opt_l2 = value != 0; return HPCCG_OK;
        case HPCCG_OPT_PDL:
            if (value < 0 || value > 2) return fail(HPCCG_EINVAL, "pdl: 0, 1 or 2");
            p->opt_pdl = value != 0;
            for (Slab &sl : p->slabs) sl.early_trigger = value == 1;
            return HPCCG_OK;
        case HPCCG_OPT_PERSISTENT:
            if (value < 0 || value > 2) return fail(HPCCG_EINVAL, "persistent: 0, 1 or 2");
            p->opt_persist = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_SMEM_SOLVE: p->opt_smem = value != 0; return HPCCG_OK;
        case HPCCG_OPT_SPMV_FORMAT:
            if (value != 0 && value != 1) return fail(HPCCG_EINVAL, "spmv format: 0 (ELL-27) or 1 (DIA-27)");
            for (Slab &sl : p->slabs) sl.dia = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_FINISHER_FREE: p->opt_ff = value != 0; return HPCCG_OK;
        case HPCCG_OPT_SERPENTINE:
            if (value < -1 || value > 3) return fail(HPCCG_EINVAL, "serpentine: bit mask 0..3 or -1 (auto)");
            p->opt_serp = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_HALO_PEER:
            if (value < 0 || value > 2) return fail(HPCCG_EINVAL, "halo peer: 0, 1 or 2");
            if (value && p->ctx->mode != MODE_SINGLE && !p->slabs[0].ptab) CHECK(enable_peer(p));
            p->opt_peer = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_SPMV_SLICED:
            if (value < -1 || value > 1) return fail(HPCCG_EINVAL, "spmv sliced: -1 (auto), 0 or 1");
            if (p->graph) cudaGraphExecDestroy(p->graph);
            if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
            p->graph = p->wgraph = nullptr;
            p->opt_sliced = (int)value;
            return sliced_alloc(p);
        case HPCCG_OPT_SMEM_HALO:
            if (value < -1 || value > 1) return fail(HPCCG_EINVAL, "smem halo: -1 (auto), 0 or 1");
            p->opt_smem_halo = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_SPMV_CLUSTER:
            if (value < -1 || value > 1) return fail(HPCCG_EINVAL, "spmv cluster: -1 (auto), 0 or 1");
            if (p->graph) cudaGraphExecDestroy(p->graph);
            if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
            p->graph = p->wgraph = nullptr;
            p->opt_spmv_cl = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_PAP_CLUSTER:
            if (value != 0 && value != 1) return fail(HPCCG_EINVAL, "pap cluster: 0 or 1");
            if (p->graph) cudaGraphExecDestroy(p->graph);
            if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
            p->graph = p->wgraph = nullptr;
            p->opt_pap_cluster = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_SPMV_TRIPS:
            if (value < 0 || value > 4096) return fail(HPCCG_EINVAL, "spmv trips: 0 (auto), 1 (off) .. 4096");
            if (p->graph) cudaGraphExecDestroy(p->graph);
            if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
            p->graph = p->wgraph = nullptr;
            p->opt_spmv_trips = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_FUSE_PSPMV:
            if (value < -1 || value > 1) return fail(HPCCG_EINVAL, "fuse pspmv: -1 (auto), 0 or 1");
            if (p->opt_fuse_ps != (int)value) {
                if (p->graph) cudaGraphExecDestroy(p->graph);
                if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
                p->graph = p->wgraph = nullptr;
            }
            p->opt_fuse_ps = (int)value;
            if (value != 0 && p->ctx->mode == MODE_SINGLE) CHECK(ps_alloc(p->slabs[0]));
            return HPCCG_OK;
        case HPCCG_OPT_PS_LEAD:
            if (value < 0 || value > (1 << 20)) return fail(HPCCG_EINVAL, "ps lead: 0 (auto) .. 2^20 chunks");
            if (p->graph) cudaGraphExecDestroy(p->graph);
            if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
            p->graph = p->wgraph = nullptr;
            p->opt_ps_lead = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_DEFER_X:
            if (value < -1 || value > kRingMaxM)
                return fail(HPCCG_EINVAL, "defer x: -1 (auto), 0, 1 or a ring depth 2 .. %d", kRingMaxM);
            if (p->opt_defer_x != (int)value) {  // graphs capture the choice
                if (p->graph) cudaGraphExecDestroy(p->graph);
                if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
                p->graph = p->wgraph = nullptr;
            }
            CHECK(ring_alloc(p, value < 0 ? (p->slabs[0].arena_bytes > ((size_t)126 << 20) ? kRingAutoM : 0)
                                          : (int)value));
            p->opt_defer_x = (int)value;
            // loopback slabs: re-address the (new) rings in the peer tables; one slab per
            // process exchanges them only at HALO_PEER setup (a collective)
            if (p->ctx->mode == MODE_LOOPBACK && p->slabs[0].ptab) CHECK(enable_peer(p));
            return HPCCG_OK;
        case HPCCG_OPT_PEER_TIMEOUT_MS:
            if (value < 1 || value > 3600000) return fail(HPCCG_EINVAL, "peer timeout: 1 .. 3600000 ms");
            p->opt_peer_timeout_ms = value;
            return peer_set_timeout(p);
        case HPCCG_OPT_SMEM_THREADS:
            if (value != 0 && value != 256 && value != 512) return fail(HPCCG_EINVAL, "smem threads: 0, 256, 512");
            p->opt_smem_threads = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_CG_VARIANT:
            if (value != 0 && value != 1) return fail(HPCCG_EINVAL, "cg variant: 0 or 1");
            p->opt_variant = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_WHILE_UNROLL:
            if (value < 1 || value > 64) return fail(HPCCG_EINVAL, "while unroll must be 1..64");
            p->opt_while_unroll = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_TRACE: {
            if (value < 0 || value > (1 << 20)) return fail(HPCCG_EINVAL, "trace: 0..2^20 iterations");
            for (Slab &sl : p->slabs) {
                cudaFree(sl.trace);
                sl.trace = nullptr;
                sl.trace_max = 0;
                sl.trace_on = false;
                if (value > 0) {
                    CHECK(alloc_zero((void **)&sl.trace, sizeof(TraceSlot) * 3 * (size_t)value));
                    sl.trace_max = (int)value;
                    sl.trace_on = true;
                }
            }
            return HPCCG_OK;
        }
        case HPCCG_OPT_CLUSTER_ROWS:
            if (value < 0) return fail(HPCCG_EINVAL, "cluster rows must be >= 0");
            p->opt_cluster_rows = value;
            return HPCCG_OK;
        case HPCCG_OPT_PERSIST_ROWS:
            if (value < -1) return fail(HPCCG_EINVAL, "persist rows must be >= 0 or -1 (auto)");
            p->opt_persist_rows = value;
            return HPCCG_OK;
        case HPCCG_OPT_VEC_UNROLL:
            if (value != 1 && value != 2 && value != 4) return fail(HPCCG_EINVAL, "unroll: 1, 2 or 4");
            p->opt_unroll = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_SPMV_ROWS:
            if (value != 1 && value != 2) return fail(HPCCG_EINVAL, "spmv rows must be 1 or 2");
            p->opt_rows = (int)value;
            return HPCCG_OK;
        case HPCCG_OPT_VEC_WAVES:
            if (value < 0 || value > 64) return fail(HPCCG_EINVAL, "vec waves must be 0..64");
            p->opt_vec_waves = (int)value;
            return HPCCG_OK;
        default: return fail(HPCCG_EINVAL, "unknown option %d", key);
    }
}

int hpccg_spmv(hpccg_problem *p, double *x, double *y) {
    if (!p || !x || !y) return fail(HPCCG_EINVAL, "NULL argument");
    hpccg_ctx *ctx = p->ctx;
    CU(cudaSetDevice(ctx->device));
    const size_t P = p->slabs.size();
    const Slab &s0 = p->slabs[0];
    std::vector<double *> xs(P);
    for (size_t i = 0; i < P; ++i) xs[i] = x + i * s0.ncol;
    // halo exchange on the main stream (API call: no overlap needed)
    CHECK(exchange(p, xs.data(), ctx->stream));
    for (size_t i = 0; i < P; ++i)
        CHECK(spmv_plain(ctx, p->opt_minb, p->opt_rows, p->slabs[i], xs[i], y + i * s0.n,
                         ctx->stream));
    CU(cudaStreamSynchronize(ctx->stream));
    return HPCCG_OK;
}

int hpccg_ddot(hpccg_ctx *ctx, int64_t n, const double *x, const double *y, double *result) {
    if (!ctx || !result || n < 0 || (n > 0 && (!x || !y))) return fail(HPCCG_EINVAL, "bad argument");
    CU(cudaSetDevice(ctx->device));
    return api_reduce(ctx, false, result, [&](int s, double *out) {
        const double *xs = x + (size_t)s * n, *ys = y + (size_t)s * n;
        const bool vec = aligned16(xs) && aligned16(ys);
        const int u = ctx->dot_unroll;
        auto k = !vec ? dot_kernel<false> : (u == 2 ? dot_kernel<true, 2> : dot_kernel<true, 4>);
        const int g = std::min<int>(wave_grid(vec ? cdiv(n, 2 * u) : n, wave(ctx, k)), (int)ctx->red_cap);
        k<<<g, kBlock, 0, ctx->stream>>>(n, xs, ys, ctx->red, out);
        return check_launch(ctx);
    });
}

int hpccg_waxpby(hpccg_ctx *ctx, int64_t n, double alpha, const double *x, double beta,
                 const double *y, double *w) {
    if (!ctx || n < 0 || (n > 0 && (!x || !y || !w))) return fail(HPCCG_EINVAL, "bad argument");
    CU(cudaSetDevice(ctx->device));
    const int64_t tot = n * ctx->nslabs;
    if (tot == 0) return HPCCG_OK;
    const bool vec = aligned16(x) && aligned16(y) && aligned16(w);
    const int u = ctx->axpy_unroll;
    const int g = wave_grid(vec ? cdiv(tot, 2 * u) : tot, wave(ctx, waxpby_kernel<true, 2, 2>));
    const int form = alpha == 1.0 ? 0 : (beta == 1.0 ? 1 : 2);
    cudaStream_t st = ctx->stream;
#define WAX(V, F, U) waxpby_kernel<V, F, U><<<g, kBlock, 0, st>>>(tot, alpha, x, beta, y, w)
    if (vec && u == 2) {
        if (form == 0) WAX(true, 0, 2); else if (form == 1) WAX(true, 1, 2); else WAX(true, 2, 2);
    } else if (vec) {
        if (form == 0) WAX(true, 0, 4); else if (form == 1) WAX(true, 1, 4); else WAX(true, 2, 4);
    } else {
        if (form == 0) WAX(false, 0, 1); else if (form == 1) WAX(false, 1, 1); else WAX(false, 2, 1);
    }
#undef WAX
    CHECK(check_launch(ctx));
    CU(cudaStreamSynchronize(st));
    return HPCCG_OK;
}

// f3: grid of 32 x 8 blocks covering m x n, capped at ~2 waves (grid-stride beyond)
static dim3 grid2d(int64_t m, int64_t n, int64_t cap_blocks) {
    int64_t gx = std::max<int64_t>(1, std::min<int64_t>(cdiv(m, kB2x), 256));
    int64_t gy = std::max<int64_t>(1, std::min<int64_t>(cdiv(n, kB2y), cap_blocks / gx));
    gy = std::max<int64_t>(1, std::min<int64_t>(gy, 65535));
    return dim3((unsigned)gx, (unsigned)gy);
}

int hpccg_waxpby2d(hpccg_ctx *ctx, int64_t m, int64_t n, int64_t ld, double alpha, const double *x,
                   double beta, const double *y, double *w) {
    if (!ctx || m < 0 || n < 0 || ld < m || (m > 0 && n > 0 && (!x || !y || !w)))
        return fail(HPCCG_EINVAL, "hpccg_waxpby2d: bad argument");
    if (m == 0 || n == 0) return HPCCG_OK;
    CU(cudaSetDevice(ctx->device));
    // a contiguous m x n array (ld == m) is the 1-D AXPY over m n elements
    // (same memory pattern, identical bits): use the vectorised 1-D kernel
    if (ld == m) return hpccg_waxpby(ctx, m * n, alpha, x, beta, y, w);
    const int form = alpha == 1.0 ? 0 : (beta == 1.0 ? 1 : 2);
    const dim3 g = grid2d(m, (int64_t)n * ctx->nslabs, 2 * 148 * 8), b(kB2x, kB2y);
    const int64_t nn = (int64_t)n * ctx->nslabs;  // loopback: slabs stacked column-wise
    if (form == 0) waxpby2d_kernel<0><<<g, b, 0, ctx->stream>>>(m, nn, ld, alpha, x, beta, y, w);
    else if (form == 1) waxpby2d_kernel<1><<<g, b, 0, ctx->stream>>>(m, nn, ld, alpha, x, beta, y, w);
    else waxpby2d_kernel<2><<<g, b, 0, ctx->stream>>>(m, nn, ld, alpha, x, beta, y, w);
    CHECK(check_launch(ctx));
    CU(cudaStreamSynchronize(ctx->stream));
    return HPCCG_OK;
}

int hpccg_ddot2d(hpccg_ctx *ctx, int64_t m, int64_t n, int64_t ld, const double *x, const double *y,
                 double *result) {
    if (!ctx || !result || m < 0 || n < 0 || ld < m || (m > 0 && n > 0 && (!x || !y)))
        return fail(HPCCG_EINVAL, "hpccg_ddot2d: bad argument");
    CU(cudaSetDevice(ctx->device));
    if (ld == m) return hpccg_ddot(ctx, m * n, x, y, result);  // contiguous: the 1-D DOT
    return api_reduce(ctx, false, result, [&](int s, double *out) {
        const double *xs = x + (size_t)s * ld * n, *ys = y + (size_t)s * ld * n;
        const dim3 g = grid2d(std::max<int64_t>(m, 1), std::max<int64_t>(n, 1),
                              std::min<int64_t>(ctx->red_cap, 2 * 148 * 8));
        dot2d_kernel<<<g, dim3(kB2x * kB2y), 0, ctx->stream>>>(m, n, ld, xs, ys, ctx->red, out);
        return check_launch(ctx);
    });
}

int hpccg_maxabsdiff(hpccg_problem *p, double *result) {
    if (!p || !result) return fail(HPCCG_EINVAL, "NULL argument");
    hpccg_ctx *ctx = p->ctx;
    CU(cudaSetDevice(ctx->device));
    if (ctx->mode == MODE_PEER) {  // local max, then the problem's peer allreduce (max)
        if (!peer_on(p)) return fail(HPCCG_EINVAL, "peer-only context: call hpccg_peer_attach");
        const Slab &sl = p->slabs[0];
        const int g = std::min<int>(wave_grid(sl.n, wave(ctx, maxabsdiff_kernel)), (int)ctx->red_cap);
        maxabsdiff_kernel<<<g, kBlock, 0, ctx->stream>>>(sl.n, sl.x, sl.xexact, ctx->red, &sl.sc->red_loc);
        CHECK(check_launch(ctx));
        double *src[1] = {&sl.sc->red_loc}, *dst[1] = {&sl.sc->red_out};
        CHECK(peer_allreduce(p, src, dst, 1, true));
        CU(cudaMemcpyAsync(ctx->h_pinned, &sl.sc->red_out, sizeof(double), cudaMemcpyDeviceToHost,
                           ctx->stream));
        CU(cudaStreamSynchronize(ctx->stream));
        CHECK(peer_check_error(p, "hpccg_maxabsdiff"));
        *result = *(volatile double *)ctx->h_pinned;
        return HPCCG_OK;
    }
    return api_reduce(ctx, true, result, [&](int s, double *out) {
        const Slab &sl = p->slabs[s];
        const int g = std::min<int>(wave_grid(sl.n, wave(ctx, maxabsdiff_kernel)), (int)ctx->red_cap);
        maxabsdiff_kernel<<<g, kBlock, 0, ctx->stream>>>(sl.n, sl.x, sl.xexact,
                                                                         ctx->red, out);
        return check_launch(ctx);
    });
}

int hpccg_solve(hpccg_problem *p, int max_iter, double tol, int *niters, double *normr,
                double times[6]) {
    if (!p) return fail(HPCCG_EINVAL, "NULL problem");
    if (max_iter < 1 || !(tol >= 0.0)) return fail(HPCCG_EINVAL, "max_iter >= 1 and tol >= 0 required");
    if (p->ctx->mode == MODE_PEER && !peer_on(p))
        return fail(HPCCG_EINVAL, "peer-only context: call hpccg_peer_attach before solving");
    hpccg_ctx *ctx = p->ctx;
    CU(cudaSetDevice(ctx->device));
    const bool timing = p->opt_timing != 0;
    const bool use_graph = p->opt_graph && !timing;
    // f2 (single-reduction) has a persistent form only on chip (smem cluster)
    const bool use_persist = !timing && ctx->mode == MODE_SINGLE &&
                             (p->opt_variant == 0 || smem_rows(p) > 0) &&
                             (p->opt_persist == 2 ||
                              (p->opt_persist == 1 && (p->opt_persist_rows < 0 ? smem_rows(p) > 0
                                                                             : p->slabs[0].n <= p->opt_persist_rows)));
    // NCCL calls cannot live in a conditional graph body; with HALO_PEER the
    // multi-GPU iteration is our own kernels only, so it can
    bool use_while = !use_persist && use_graph && p->opt_while && (ctx->mode != MODE_NCCL || peer_on(p)) &&
                     !p->while_failed;
    p->ev_used = 0;
    p->timed.clear();
    // a slab whose earlier peer wait timed out has lost step with its peers (the
    // flag counts / epochs no longer agree): refuse to run instead of computing on
    // stale halos (the peers then time out too and report it)
    if (peer_on(p) && peer_check_error(p, "hpccg_solve") != HPCCG_OK) {
        const std::string why = g_err;
        return fail(HPCCG_ECUDA, "%s -- an earlier solve of this problem timed out: recreate it "
                    "(hpccg_free + hpccg_generate)", why.c_str());
    }
    const int64_t l0 = ctx->launches;
    // the persisting-L2 window costs two device-limit changes per solve; the
    // persistent kernels keep their small working set on chip / in L2 anyway
    L2Window l2win(p, !use_persist);
    if (use_while && build_while_graph(p, max_iter, tol) != HPCCG_OK) {
        p->while_failed = true;  // keep the message in hpccg_last_error; fall back
        use_while = false;
    }
    if (use_graph && !use_while && !use_persist) CHECK(build_graph(p));

    if (p->slabs[0].trace_on) {  // t0 = +inf, t1 = 0 for every slot
        const Slab &s0 = p->slabs[0];
        std::vector<TraceSlot> init((size_t)3 * s0.trace_max, TraceSlot{~0ull, 0ull});
        CU(cudaMemcpyAsync(s0.trace, init.data(), sizeof(TraceSlot) * init.size(),
                           cudaMemcpyHostToDevice, ctx->stream));
        CU(cudaStreamSynchronize(ctx->stream));
    }
    CU(cudaEventRecord(p->ev_t0, ctx->stream));
    if (use_persist) {
        CHECK(launch_persistent(p, max_iter, tol));
    } else if (use_while) {
        CU(cudaGraphLaunch(p->wgraph, ctx->stream));
    } else {
        CHECK(enqueue_init_any(p, max_iter, tol, timing, 0ull));
        // at most max_iter - 1 iterations (A4); finished iterations turn the
        // remaining launches into no-ops on the device (done flag)
        const int per_graph = body_iterations(p, 1);
        const int64_t iters = (int64_t)max_iter - 1;
        const int poll = (tol > 0.0) ? p->opt_poll : 0;
        const int *d_done = &p->slabs[0].sc->done;
        int64_t launched = 0;
        int chunk = 0;
        bool stop = false;
        while (launched < iters && !stop) {
            const int64_t m = poll > 0 ? std::min<int64_t>(poll, iters - launched) : iters - launched;
            int64_t i = 0;
            while (i < m) {
                if (use_graph) {  // per_graph iterations per replay
                    CU(cudaGraphLaunch(p->graph, ctx->stream));
                    ctx->launches += p->graph_kernels;
                    i += per_graph;
                } else {
                    CHECK(enqueue_iteration_any(p, timing, true, 0ull, (int)(launched + i + 1)));
                    ++i;
                }
            }
            launched += i;
            if (poll > 0 && launched < iters) {
                // double-buffered poll: queue this chunk's flag copy, then look at
                // the previous chunk's, so the GPU always has a chunk queued
                const int slot = chunk & 1;
                CU(cudaMemcpyAsync(&p->h_done[slot], d_done, sizeof(int), cudaMemcpyDeviceToHost,
                                   ctx->stream));
                CU(cudaEventRecord(p->ev_poll[slot], ctx->stream));
                if (chunk > 0) {
                    CU(cudaEventSynchronize(p->ev_poll[slot ^ 1]));
                    if (p->h_done[slot ^ 1]) stop = true;
                }
                ++chunk;
            }
        }
        CHECK(enqueue_xfix(p));
    }
    CU(cudaEventRecord(p->ev_t1, ctx->stream));
    // the loop state comes back in the same synchronisation as the solve
    if (!p->h_sc) CU(cudaMallocHost((void **)&p->h_sc, sizeof(CgScalars)));
    CU(cudaMemcpyAsync(p->h_sc, p->slabs[0].sc, sizeof(CgScalars), cudaMemcpyDeviceToHost, ctx->stream));
    CU(cudaStreamSynchronize(ctx->stream));
    CU(cudaGetLastError());
    l2win.release();
    if (peer_on(p)) CHECK(peer_check_error(p, "hpccg_solve"));
    for (const Slab &sl : p->slabs)
        if (sl.ps_err) {
            int e = 0;
            CU(cudaMemcpy(&e, sl.ps_err, sizeof e, cudaMemcpyDeviceToHost));
            if (e) {
                CU(cudaMemset(sl.ps_err, 0, sizeof e));
                return fail(HPCCG_ECUDA, "fused p update + SpMV: a chunk wait gave up after 5 s (residency)");
            }
        }

    const CgScalars hs = *p->h_sc;
    hpccg_stats st{};
    float ms = 0.f;
    CU(cudaEventElapsedTime(&ms, p->ev_t0, p->ev_t1));
    st.total_ms = ms;
    for (const TimedOp &t : p->timed) {
        float e = 0.f;
        if (cudaEventElapsedTime(&e, t.a, t.b) != cudaSuccess) continue;
        switch (t.phase) {
            case PH_PUPDATE: st.pupdate_ms += e; break;
            case PH_SPMV: st.spmv_ms += e; break;
            case PH_UPDATE: st.update_ms += e; break;
            case PH_ALLREDUCE: st.allreduce_ms += e; break;
            case PH_EXCHANGE: st.exchange_ms += e; break;
        }
    }
    if (use_while) ctx->launches += p->wgraph_init_kernels + p->wgraph_body_kernels * hs.niters;
    st.iterations = hs.niters;
    st.spmv_launches = hs.niters + (p->opt_variant == 1 ? 2 : 1);
    st.kernel_launches = ctx->launches - l0;
    st.l2_persist_bytes = (int64_t)l2win.kept;
    st.graph_mode = use_persist ? p->last_persist_mode : (use_while ? 2 : (use_graph ? 1 : 0));
    st.x_deferred = use_persist ? 0 : (p->opt_variant == 1 ? sr_ring_m(p) : defer_m(p));
    st.ps_fused = !use_persist && fuse_ps_on(p);
    p->stats = st;
    if (niters) *niters = hs.niters;
    if (normr) *normr = hs.normr;
    if (times) {
        times[0] = st.total_ms * 1e-3;
        times[1] = 0.0;
        times[2] = (st.pupdate_ms + st.update_ms) * 1e-3;
        times[3] = st.spmv_ms * 1e-3;
        times[4] = st.allreduce_ms * 1e-3;
        times[5] = st.exchange_ms * 1e-3;
    }
    return HPCCG_OK;
}

int hpccg_get_trace(const hpccg_problem *p, uint64_t *out, int64_t k) {
    if (!p || !out || k < 0) return fail(HPCCG_EINVAL, "bad argument");
    const Slab &s = p->slabs[0];
    if (!s.trace_on) return fail(HPCCG_EINVAL, "tracing is off (HPCCG_OPT_TRACE)");
    const int64_t m = std::min<int64_t>(k, s.trace_max);
    CU(cudaSetDevice(p->ctx->device));
    CU(cudaMemcpy(out, s.trace, sizeof(TraceSlot) * 3 * (size_t)m, cudaMemcpyDeviceToHost));
    for (int64_t i = 0; i < 6 * m; i += 2)
        if (out[i] == ~0ull) out[i] = out[i + 1] = 0;  // kernel did not run
    return HPCCG_OK;
}

int hpccg_get_stats(const hpccg_problem *p, hpccg_stats *out) {
    if (!p || !out) return fail(HPCCG_EINVAL, "NULL argument");
    *out = p->stats;
    return HPCCG_OK;
}

void hpccg_free(hpccg_problem *p) {
    if (!p) return;
    cudaSetDevice(p->ctx->device);
    cudaStreamSynchronize(p->ctx->stream);
    if (p->graph) cudaGraphExecDestroy(p->graph);
    if (p->wgraph) cudaGraphExecDestroy(p->wgraph);
    for (void *q : p->ipc_opened) cudaIpcCloseMemHandle(q);
    for (Slab &s : p->slabs) free_slab(s);
    cudaFree(p->d_tab);
    for (cudaEvent_t e : p->ev_pool) cudaEventDestroy(e);
    if (p->ev_t0) cudaEventDestroy(p->ev_t0);
    if (p->ev_t1) cudaEventDestroy(p->ev_t1);
    if (p->ev_poll[0]) cudaEventDestroy(p->ev_poll[0]);
    if (p->ev_poll[1]) cudaEventDestroy(p->ev_poll[1]);
    if (p->h_done) cudaFreeHost(p->h_done);
    if (p->h_sc) cudaFreeHost(p->h_sc);
    delete p;
}

}  // extern "C"

#include "tridiag_host.inc"
#include "lbm_host.inc"
