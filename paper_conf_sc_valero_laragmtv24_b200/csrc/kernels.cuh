// kernels.cuh -- sm_100a device code of the HPCCG CG hot path.
//
// Every step of the path runs here: problem generation (a.1), the 27-point
// ELL SpMV with the p.Ap epilogue (a.3, a.4), the fused x/r update + r.r
// (a.5), the p update (a.6), init (a.7), device-side loop control (a.8),
// max|x - x_exact| (a.9) and the BLAS-1 waxpby / ddot (a.10).
// Step ids and readings A<k> refer to DESIGN.md.
//
// The path is HBM-bandwidth bound (SpMV ~0.16 flop/B, BLAS-1 1/12..1/8
// flop/B): no tensor cores.  What matters is coalescing (slot-major ELL,
// consecutive rows on consecutive lanes), memory-level parallelism (all 54
// matrix loads of a row issued before the FMA chain), keeping the matrix
// stream from evicting the x planes out of L1/L2 (L1::no_allocate +
// L2 evict_first on the matrix, default caching on x), and scalars that
// never leave the device.
#pragma once

#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace hpccg {

constexpr int kSlots = 27;      // 3x3x3 stencil slots per ELL row
constexpr int kDiagSlot = 13;   // (sz, sy, sx) = (0, 0, 0)
constexpr int kBlock = 256;     // threads per block of every kernel
constexpr int kWarps = kBlock / 32;

// Device-resident CG state, one per slab (A4 loop semantics, DESIGN.md
// "Device-side scalars").  rr_cur / rr_prev are GLOBAL (allreduced) values.
struct CgScalars {
    double rr_cur;    // r.r of the current r            (global)
    double rr_prev;   // rtrans of the previous iteration (global)
    double pAp;       // p.Ap of this iteration           (global)
    double loc_rr;    // this slab's partial r.r   (allreduce input)
    double loc_pAp;   // this slab's partial p.Ap  (allreduce input)
    double normr;     // sqrt(rtrans) of the last iteration run
    double tol;
    double red_loc;   // generic reduction (ddot API, maxabsdiff): local
    double red_out;   //   ... and global result
    unsigned long long nnz;  // stored entries counted by gen27
    int k;            // index of the next CG iteration
    int niters;
    int done;         // loop-exit flag, read by every CG kernel
    int max_iter;
    // f2 single-reduction CG (HPCCG_OPT_CG_VARIANT = 1).  Double-buffered by
    // iteration parity q = k & 1: the update of iteration k reads slot q^1
    // (written by iteration k-1, or by init for k = 1) and its block 0 writes
    // slot q, so no block ever reads a slot another block of the same grid
    // writes.
    double sr_gamma[2];   // gamma_(k-1) = r_(k-1).r_(k-1) (global)
    double sr_alpha[2];   // alpha_k
    double gd[2];         // global (gamma, delta) when not summed from partials
    double loc_gd[2];     // this slab's (gamma, delta) partial (allreduce input)
    int sr_k[2];          // index of the next iteration
    int run_q[2];         // run_q[q]: iteration k + 1 runs (written by iteration k);
                          // also used by HPCCG's finisher-free single-slab loop
    unsigned long long epoch;  // solves initialised so far (HALO_PEER = 2 tags)
    double alpha_x;   // deferred x update: alpha of the last x/r update (x += alpha_x p
                      // is applied by the next p update, or by cg_xfix_kernel at the end)
    // deferred x update over a ring of p buffers (HPCCG_OPT_DEFER_X = m >= 2):
    // alpha_k of every x/r update (slot k & 15), and the index of the last p
    // update that ran, double-buffered by iteration parity (ring_k[q] written
    // by p update k, q = k & 1; read by p update k + 1 before its PDL wait)
    double alpha_h[16];
    int ring_k[2];
};

// Scratch for the deterministic single-pass grid reduction.
struct Reduction {
    double *partials;       // one slot per block (of all launches in the pass)
    unsigned int *counter;  // blocks finished; reset to 0 by the last block
};

// ------------------------------------------------------------ PTX helpers

__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// Matrix stream: read once per SpMV -> do not allocate in L1, evict first
// from L2 so it does not push the x planes / CG vectors out.
__device__ __forceinline__ double ld_stream(const double *ptr, uint64_t pol) {
    double v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;"
        : "=d"(v) : "l"(ptr), "l"(pol));
    return v;
}

__device__ __forceinline__ int ld_stream(const int *ptr, uint64_t pol) {
    int v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;"
        : "=r"(v) : "l"(ptr), "l"(pol));
    return v;
}

// 16-B / 8-B vector forms for two adjacent rows (slot-major: same slot)
__device__ __forceinline__ double2 ld_stream2(const double *ptr, uint64_t pol) {
    double2 v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;"
        : "=d"(v.x), "=d"(v.y) : "l"(ptr), "l"(pol));
    return v;
}

__device__ __forceinline__ int2 ld_stream2(const int *ptr, uint64_t pol) {
    int2 v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.s32 {%0, %1}, [%2], %3;"
        : "=r"(v.x), "=r"(v.y) : "l"(ptr), "l"(pol));
    return v;
}

// L2 retention hints on the CG loop's vector stores (HPCCG_STORE_HINTS): bit 0
// p (ring p update), bit 1 Ap (CG SpMV), bit 2 r (x/r update) stored with an L2
// evict_last policy, so the next kernel's reads of them hit L2.  Default 5 (p
// and r): measured at 256^3 (profiles/r2_store_hints_ab.log, one box, two
// runs) period 929.3 / 929.8 -> 923.4 / 923.1 us (p alone 924.8, p + Ap 927,
// all three 926: Ap kept in L2 costs the next SpMV more than the update gains);
// 128^3 (vectors L2-resident) unchanged
#ifndef HPCCG_STORE_HINTS
#define HPCCG_STORE_HINTS 5
#endif
template <int kBit>
__device__ __forceinline__ void st_hint(double2 *p, double2 v) {
    if (HPCCG_STORE_HINTS & kBit) {
        uint64_t pol;
        asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
        asm volatile("st.global.L2::cache_hint.v2.f64 [%0], {%1, %2}, %3;" ::"l"(p), "d"(v.x), "d"(v.y), "l"(pol)
                     : "memory");
    } else {
        *p = v;
    }
}
__device__ __forceinline__ void st_p(double2 *p, double2 v) { st_hint<1>(p, v); }
// loads with an L2 evict_first policy when bit kBit of HPCCG_STORE_HINTS is set
// (bit 3: the ring p update's r and p_(K-1); bit 4: the x/r update's Ap)
template <int kBit>
__device__ __forceinline__ double2 ld_hint(const double2 *p) {
    if (HPCCG_STORE_HINTS & kBit) {
        uint64_t pol;
        asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
        double2 v;
        asm volatile("ld.global.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;" : "=d"(v.x), "=d"(v.y) : "l"(p), "l"(pol));
        return v;
    }
    return *p;
}

// Loads of data the PREDECESSOR grid wrote (device scalars, reduction
// partials), after pdl_wait().  ldg_o: the read-only path (one L2 request per
// SM serves every warp; plain loads cost 1.6 % at 128^3).  The compiler may
// hoist an ld.global.nc above griddepcontrol.wait (SASS ACQBULK) -- the nc
// contract says the data is constant for the kernel's lifetime -- and did so
// in the fused p update + SpMV kernel, which therefore uses plain loads (ldp);
// tests/test_abi_cpu.py fails the build if any kernel's SASS has a read-only
// load ahead of its first ACQBULK.
__device__ __forceinline__ double ldg_o(const double *p) { return __ldg(p); }
__device__ __forceinline__ int ldg_o(const int *p) { return __ldg(p); }
__device__ __forceinline__ unsigned long long ldg_o(const unsigned long long *p) { return __ldg(p); }
template <class T>
__device__ __forceinline__ T ldp(const T *p) { return *p; }  // plain weak load (never nc)

// Programmatic dependent launch (PDL): a kernel launched with the
// programmatic-stream-serialization attribute may start while its
// predecessor drains; pdl_wait() (griddepcontrol.wait) blocks until the
// predecessor grid has completed and its writes are visible, and is a no-op
// for an ordinary launch.  pdl_trigger() lets the successor be scheduled.
// Before pdl_wait() a kernel may only read data no in-flight predecessor
// writes (the matrix).
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;"); }

// Device-side trace (HPCCG_OPT_TRACE): for traced iteration k and CG kernel j
// (0 p update, 1 SpMV, 2 x/r update) the earliest block start and the latest
// block end on %globaltimer (ns), so per-kernel times and the gaps between
// kernels can be read even inside the while-graph (no events allowed there).
struct TraceSlot {
    unsigned long long t0, t1;
};

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ void trace_mark(TraceSlot *tr, int trace_max, int k, int j, bool end) {
    if (!tr || threadIdx.x != 0 || k < 1 || k > trace_max) return;
    TraceSlot *s = tr + (size_t)(k - 1) * 3 + j;
    if (end) atomicMax(&s->t1, gtimer());
    else atomicMin(&s->t0, gtimer());
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

__device__ __forceinline__ double warp_max(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmax(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

// Block-wide reduction in a fixed order (butterfly per warp, then warp 0 over
// the per-warp values).  Result valid in every thread of warp 0.
template <bool kMax>
__device__ __forceinline__ double block_reduce(double v, double *sh) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    __syncwarp();  // reconverge lanes that left a grid-stride loop at different trips
    v = kMax ? warp_max(v) : warp_sum(v);
    if (lane == 0) sh[warp] = v;
    __syncwarp();  // converged warp at the block barrier (compute-sanitizer synccheck)
    __syncthreads();
    if (warp == 0) {
        v = (lane < kWarps) ? sh[lane] : (kMax ? 0.0 : 0.0);
        v = kMax ? warp_max(v) : warp_sum(v);
    }
    return v;
}

// Deterministic single-pass grid reduction ("last block done"): every block
// writes its partial to partials[part]; the block that finishes last sums all
// `total` partials in a fixed order and calls fin(result) on thread 0.  The
// result depends only on the grid shape, never on scheduling (no fp atomics).
// kMax: max instead of sum (values are >= 0).
template <bool kMax, class Fin>
__device__ __forceinline__ void grid_reduce(double v, Reduction red, unsigned part,
                                            unsigned total, Fin fin) {
    __shared__ double sh[32];
    __shared__ int is_last;
    v = block_reduce<kMax>(v, sh);
    if (threadIdx.x == 0) {
        red.partials[part] = v;
        __threadfence();
        unsigned t = atomicAdd(red.counter, 1u);
        is_last = (t == total - 1);
    }
    __syncwarp();
    __syncthreads();
    if (!is_last) return;
    __threadfence();
    double s = 0.0;
    for (unsigned i = threadIdx.x; i < total; i += kBlock) {
        double q = __ldcg(red.partials + i);
        s = kMax ? fmax(s, q) : s + q;
    }
    __syncthreads();  // sh reuse
    s = block_reduce<kMax>(s, sh);
    if (threadIdx.x == 0) {
        *red.counter = 0u;
        fin(s);
    }
}

// ------------------------------------------------------- a.1 generation

struct GenArgs {
    int nx, ny, nz;       // local slab dims
    int rank, nranks;     // z-slab of the global nx x ny x (nz*nranks) grid
    int64_t n, plane;     // rows, nx*ny
    double *val;          // [27][n]
    int *col;             // [27][n]  local-with-halo index
    double *b, *x, *xexact;
    unsigned long long *nnz;
};

// One thread per local row.  Slot s <-> (sz, sy, sx) = (s/9-1, s/3%3-1, s%3-1):
// ascending column (A8).  Absent neighbour -> padding (0.0, own column).
__global__ void __launch_bounds__(kBlock) gen27_kernel(GenArgs a) {
    __shared__ double sh[32];
    const int64_t i = (int64_t)blockIdx.x * kBlock + threadIdx.x;
    double cnt_d = 0.0;
    if (i < a.n) {
        const int64_t iz = i / a.plane;
        const int64_t rem = i - iz * a.plane;
        const int iy = (int)(rem / a.nx);
        const int ix = (int)(rem - (int64_t)iy * a.nx);
        const int64_t gz = (int64_t)a.rank * a.nz + iz;
        const int64_t nzg = (int64_t)a.nz * a.nranks;
        const int64_t own = i + a.plane;  // local-with-halo index of row i
        int cnt = 0;
#pragma unroll
        for (int s = 0; s < kSlots; ++s) {
            const int sz = s / 9 - 1, sy = (s / 3) % 3 - 1, sx = s % 3 - 1;
            const bool in = (ix + sx >= 0) && (ix + sx < a.nx) && (iy + sy >= 0) &&
                            (iy + sy < a.ny) && (gz + sz >= 0) && (gz + sz < nzg);
            const int64_t c = own + sz * a.plane + (int64_t)sy * a.nx + sx;
            a.val[(int64_t)s * a.n + i] = in ? (s == kDiagSlot ? 27.0 : -1.0) : 0.0;
            a.col[(int64_t)s * a.n + i] = (int)(in ? c : own);
            cnt += in;
        }
        a.b[i] = 28.0 - (double)cnt;  // = row sum: A.1 = b, x_exact = 1
        a.x[i] = 0.0;
        a.xexact[i] = 1.0;
        cnt_d = (double)cnt;
    }
    // exact integer count (<= 27*256 per block)
    double bs = block_reduce<false>(cnt_d, sh);
    if (threadIdx.x == 0) atomicAdd(a.nnz, (unsigned long long)bs);
}

// ------------------------------- peer-memory z-slab exchange: shared state
// (protocol: see "peer-memory z-slab exchange (HALO_PEER)" below)

constexpr int kMaxPeers = 64;

struct PeerSync {                      // one per slab, in that slab's device memory
    unsigned long long flag_from_lo;   // exchanges pushed to me by rank - 1
    unsigned long long flag_from_hi;   //   ... by rank + 1
    unsigned long long recv_count;     // exchanges I have waited for
    unsigned long long push_count;     // exchanges I have pushed
    unsigned long long ar_count;       // allreduces I have collected
    unsigned long long ar_posted;      // allreduces I have posted
    unsigned int push_ticket;          // blocks of the current push done
    int error;                         // != 0: a wait timed out (PEER_WAIT_* of the first one)
    int error_peer;                    //   ... the rank it waited for
    unsigned long long timeout_ns;     // give up a wait after this long (host-set; 0 = 30 s)
    unsigned long long ar_tag[2][kMaxPeers];
    double ar_val[2][kMaxPeers][2];
    // HALO_PEER = 2 (collectives fused into the CG kernels): separate words,
    // tagged tag(epoch, seq) = epoch << 32 | seq instead of counted
    unsigned long long fflag_from_lo;  // p pushed to me by rank - 1 (seq = k)
    unsigned long long fflag_from_hi;  //   ... by rank + 1
    unsigned int fpush_ticket;         // blocks of the current fused push done
    unsigned int pad_;
    // allreduce slots, LL style: slot q (1: p.Ap, seq 2k-1; 0: r.r, seq 2k),
    // rank r: two 8-B words {32 value bits | 32-bit tag}, each single-copy
    // atomic, so a reader that sees the tag in both has the value -- no fence
    // on the post or the collect (the scalar allreduces are on the critical
    // path of every iteration; the halo flags are hidden behind the interior)
    unsigned long long fll[2][kMaxPeers][2];
    unsigned long long fll2[2][kMaxPeers][2];  // f2: delta beside gamma (in fll), seq = k
};

struct PeerTab {                       // device copy per slab; pointers may be peers'
    int rank, nranks;
    double *halo_to_lo;                // rank-1's upper halo plane (gets my first owned plane)
    double *halo_to_hi;                // rank+1's lower halo plane (gets my last owned plane)
    // ring-deferred x update (HPCCG_OPT_DEFER_X >= 2): the same planes in slot 1
    // of the neighbours' p rings (slot j >= 1: + (j - 1) ring_stride); null: no ring
    double *ring_to_lo, *ring_to_hi;
    PeerSync *mine, *lo, *hi;
    PeerSync *all[kMaxPeers];          // every rank's PeerSync (allreduce posts)
};

__device__ __forceinline__ void st_release_sys(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// what a timed-out wait was waiting for (PeerSync::error; hpccg_solve names it)
enum : int { PEER_WAIT_HALO_LO = 1, PEER_WAIT_HALO_HI = 2, PEER_WAIT_ALLREDUCE = 3, PEER_WAIT_SCALAR = 4 };

__device__ __forceinline__ unsigned long long peer_timeout_ns(const PeerSync *m) {
    const unsigned long long t = *(const volatile unsigned long long *)&m->timeout_ns;
    return t ? t : 30000000000ull;
}

// record the FIRST timeout of this slab (what, peer rank); later waits see it and return at once
__device__ __forceinline__ void peer_fail(PeerSync *m, int what, int peer) {
    if (atomicCAS(&m->error, 0, what) == 0) m->error_peer = peer;
}

// spin until *flag >= target; false (and the error record) after timeout_ns
__device__ __forceinline__ bool spin_until(const unsigned long long *flag, unsigned long long target,
                                           PeerSync *mine, int what, int peer) {
    if (ld_acquire_sys(flag) >= target) return true;  // the common case: one load
    if (*(volatile int *)&mine->error) return false;  // an earlier wait timed out: do not hang again
    const unsigned long long t0 = gtimer(), lim = peer_timeout_ns(mine);
    while (ld_acquire_sys(flag) < target) {
        if (gtimer() - t0 > lim) {
            peer_fail(mine, what, peer);
            return false;
        }
        __nanosleep(64);
    }
    return true;
}

// ---- HALO_PEER = 2: the exchange and the scalar allreduces fused into the
// finisher-free CG kernels (no push / wait / allreduce kernels, no comm
// stream, no grid-wide finisher):
//   p update k   every block sums the slab's r.r(k-1) partials (fixed order),
//                block 0 posts that to every rank, every block collects the P
//                posts (rank order) -> beta; p = r + beta p, with the first /
//                last owned plane stored straight into the neighbours' halo
//                planes as it is computed; the blocks that pushed fence and
//                take a ticket, the last raises the neighbours' flags
//   SpMV k       interior row blocks first; the boundary blocks (last in
//                block order) wait for the flags, then gather the halo with
//                L2-coherent loads; per-block p.Ap partials only
//   update k     as the p update for p.Ap (slot 1) -> alpha; r.r partials
// Halo flags carry tag(epoch, k) (monotone: the epoch, counted by the init
// kernel of every solve, is the same on every slab) and are released after a
// system-scope fence (they are off the critical path: the interior rows hide
// them).  The scalar posts are LL-style words {32 value bits | 32-bit tag}
// (ll_tag: epoch and seq = 2k - 1 for p.Ap, 2k for r.r) that need no fence
// -- the two allreduces sit on the critical path of every iteration.  Slots
// alternate by seq parity; a rank cannot post seq m + 2 before every rank
// has collected m (the post follows its own collect of m + 1, which needs
// everyone's post of m + 1, made after their collect of m).  A push of
// iteration k + 1 follows the collect of r.r(k), whose posts depend on the
// neighbours' SpMV k results (so on their halo reads).  The local sums use
// the last-block finisher's order and the rank-order sums are those of
// peer_allreduce_kernel: bit-identical to HALO_PEER = 1 and the loopback copies.
__device__ __forceinline__ unsigned long long ftag(unsigned long long epoch, unsigned long long seq) {
    return (epoch << 32) | seq;
}

// 32-bit tag of the LL slots: bit 31 set (never the zero of a fresh slot),
// 11 bits of the epoch, 20 of seq.  A stale word could only match after 2048
// solves that never rewrote the slot.
__device__ __forceinline__ unsigned ll_tag(unsigned long long epoch, unsigned long long seq) {
    return 0x80000000u | ((unsigned)(epoch & 0x7FFu) << 20) | (unsigned)(seq & 0xFFFFFu);
}

// post v as rank t->rank into slot q of every rank (one thread)
__device__ __forceinline__ void fused_post(const PeerTab *t, int q, double v, unsigned tag) {
    const unsigned long long b = (unsigned long long)__double_as_longlong(v);
    const unsigned long long hi = (unsigned long long)tag << 32;
    const unsigned long long w0 = (b & 0xffffffffull) | hi, w1 = (b >> 32) | hi;
    const int P = t->nranks, me = t->rank;
    for (int r = 0; r < P; ++r)
        asm volatile("st.relaxed.sys.global.v2.u64 [%0], {%1, %2};" ::"l"(&t->all[r]->fll[q][me][0]),
                     "l"(w0), "l"(w1)
                     : "memory");
}

__device__ __forceinline__ bool ll_read(const unsigned long long *w, unsigned tag, double *v) {
    unsigned long long a, b;
    asm volatile("ld.relaxed.sys.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(w) : "memory");
    if ((unsigned)(a >> 32) != tag || (unsigned)(b >> 32) != tag) return false;
    *v = __longlong_as_double((long long)((a & 0xffffffffull) | (b << 32)));
    return true;
}

// wait for the P posts of slot q and sum them in rank order; the block's
// result (*sh broadcasts it).  Lane r of warp 0 polls rank r's words (the P
// latencies overlap); lane 0 adds the shuffled values left to right (the
// order of peer_allreduce_kernel).  ~2 s timeout -> error flag.
// `mine`: this slab's own value (every block holds it), used for slot [rank]
// instead of waiting for its own block 0's post -- same bits.
__device__ __forceinline__ double fused_collect_block(const PeerTab *t, int q, unsigned tag, double mine,
                                                      double *sh) {
    __syncthreads();  // sh reuse
    if (threadIdx.x < 32) {
        PeerSync *m = t->mine;
        const int P = t->nranks, lane = threadIdx.x;
        double s = 0.0;
        for (int r0 = 0; r0 < P; r0 += 32) {
            double v = mine;
            if (r0 + lane < P && r0 + lane != t->rank && !ll_read(m->fll[q][r0 + lane], tag, &v)) {
                const unsigned long long t0 = gtimer(), lim = peer_timeout_ns(m);
                while (!ll_read(m->fll[q][r0 + lane], tag, &v)) {
                    if (*(volatile int *)&m->error) break;
                    if (gtimer() - t0 > lim) {
                        peer_fail(m, PEER_WAIT_SCALAR, r0 + lane);
                        break;
                    }
                    __nanosleep(32);
                }
            }
            for (int j = 0; j < 32 && r0 + j < P; ++j) {
                const double w = __shfl_sync(0xffffffffu, v, j);
                s = (r0 + j == 0) ? w : s + w;
            }
        }
        if (lane == 0) *sh = s;
    }
    __syncthreads();
    return *sh;
}

// f2 (HALO_PEER = 2): (gamma, delta) of one iteration in slot q = seq & 1 of
// fll (gamma) and fll2 (delta); post by one thread, collect per block as above
__device__ __forceinline__ void fused_post2(const PeerTab *t, int q, double2 v, unsigned tag) {
    const unsigned long long hi = (unsigned long long)tag << 32;
    const unsigned long long g = (unsigned long long)__double_as_longlong(v.x);
    const unsigned long long d = (unsigned long long)__double_as_longlong(v.y);
    const int P = t->nranks, me = t->rank;
    for (int r = 0; r < P; ++r) {
        asm volatile("st.relaxed.sys.global.v2.u64 [%0], {%1, %2};" ::"l"(&t->all[r]->fll[q][me][0]),
                     "l"((g & 0xffffffffull) | hi), "l"((g >> 32) | hi)
                     : "memory");
        asm volatile("st.relaxed.sys.global.v2.u64 [%0], {%1, %2};" ::"l"(&t->all[r]->fll2[q][me][0]),
                     "l"((d & 0xffffffffull) | hi), "l"((d >> 32) | hi)
                     : "memory");
    }
}

__device__ __forceinline__ double2 fused_collect2_block(const PeerTab *t, int q, unsigned tag, double2 mine,
                                                        double *sh /*[2]*/) {
    __syncthreads();  // sh reuse
    if (threadIdx.x < 32) {
        PeerSync *m = t->mine;
        const int P = t->nranks, lane = threadIdx.x;
        double sg = 0.0, sd = 0.0;
        for (int r0 = 0; r0 < P; r0 += 32) {
            double g = mine.x, d = mine.y;
            const int src = r0 + lane;
            if (src < P && src != t->rank) {
                const unsigned long long t0 = gtimer(), lim = peer_timeout_ns(m);
                bool okg = false, okd = false;
                while (!(okg = okg || ll_read(m->fll[q][src], tag, &g)) |
                       !(okd = okd || ll_read(m->fll2[q][src], tag, &d))) {
                    if (*(volatile int *)&m->error) break;
                    if (gtimer() - t0 > lim) {
                        peer_fail(m, PEER_WAIT_SCALAR, src);
                        break;
                    }
                    __nanosleep(32);
                }
            }
            for (int j = 0; j < 32 && r0 + j < P; ++j) {
                const double wg = __shfl_sync(0xffffffffu, g, j), wd = __shfl_sync(0xffffffffu, d, j);
                sg = (r0 + j == 0) ? wg : sg + wg;
                sd = (r0 + j == 0) ? wd : sd + wd;
            }
        }
        if (lane == 0) {
            sh[0] = sg;
            sh[1] = sd;
        }
    }
    __syncthreads();
    return make_double2(sh[0], sh[1]);
}

// --------------------------------------------------------- a.3 SpMV (ELL-27)

// Rows of up to two disjoint ranges [r0, r0+len0) and [r1, r1+len1) (the
// interior / boundary split used to overlap the halo exchange).
struct SpmvArgs {
    int64_t r0, len0, r1, len1;
    int64_t nb0;            // blocks covering range 0
    int64_t r2, len2;       // a third range (HALO_PEER = 2: interior, plane 0, plane nz-1)
    int64_t nb01;           // blocks covering ranges 0 and 1
    int64_t stride;         // slot stride = n
    int64_t plane;          // x[row + plane] is the row's own entry
    const double *val;
    const int *col;
    const double *x;        // local-with-halo base (ncol entries)
    double *y;              // n entries
    // CG epilogue (kDot): partial p.Ap -> scalars
    CgScalars *sc;
    Reduction red;
    unsigned part_base, total_blocks;
    int single;             // 1: write the global pAp directly (no allreduce)
    // single slab: write the per-block p.Ap partials here and skip the
    // last-block finisher (its fence + ticket costs ~6 us per SpMV on B200);
    // the update kernel sums the partials itself.  nullptr: finisher.
    double *parts_only;
    TraceSlot *trace;  // HPCCG_OPT_TRACE (nullptr: off)
    int trace_max;
    int sr_q;          // kDots 2: parity of the iteration (run flag run_q[sr_q])
    int early_trigger; // PDL: let the successor be scheduled right after pdl_wait
                       // (it may then prefetch its inputs that this grid does not
                       // write during this grid's tail); 0: after the rows
    const PeerTab *fpeer;  // HALO_PEER = 2 (spmv27x2_kernel<., ., true>): blocks of ranges
                           // 1 and 2 wait for the halo flags; the finisher posts p.Ap
    int rev;           // 1: block b takes the rows (and the partial slot) of block
                       // gridDim - 1 - b, i.e. the grid walks the rows backwards
                       // (same rows per block, same partials: identical bits)
    int nx;            // kDia (HPCCG_OPT_SPMV_FORMAT 1): row stride of the grid
    int dia;           // 1: spmv27x2_kernel<., ., false, true> (DIA-27, col[] not read)
    int trips;         // spmv27x2_trips_kernel: 512-row trips per block (one partial per block)
    // HPCCG_OPT_DEFER_X = m >= 2: p_k lives in ring slot k % ring_n (slot 0 =
    // x, slot j > 0 = ring + (j - 1) ring_stride), k = sc->k read after the
    // PDL wait; ring_n <= 1: x.  (Kept last: inserted after r0..len1 the field
    // offsets made ptxas spill 8 B in spmv27x2_kernel<1, true>, 95.2 -> 97.8 us
    // at 128^3)
    const double *ring;
    int64_t ring_stride;
    int ring_n;
};

// the row block this CTA handles (HPCCG_OPT_SERPENTINE)
__device__ __forceinline__ int64_t spmv_bid(const SpmvArgs &a) {
    return a.rev ? (int64_t)gridDim.x - 1 - blockIdx.x : (int64_t)blockIdx.x;
}

template <int kDots, bool kCheck>
__device__ __forceinline__ int spmv_done(const SpmvArgs &a) {
    if (!kCheck || kDots == 0) return 0;
    if (kDots == 2) return !ldg_o(&a.sc->run_q[a.sr_q]);
    return ldg_o(&a.sc->done);
}

// the gathered vector of this SpMV (after pdl_wait: sc->k is the predecessor's).
// kRing = false: a.x, no load -- the 2-rows/thread kernels instantiate the ring
// separately (the extra live pointer made the fused z-slab kCheck variant spill
// at 64 registers: 812.8 -> 853.0 us at 256^3)
template <bool kRing = true>
__device__ __forceinline__ const double *spmv_xg(const SpmvArgs &a) {
    if (!kRing || a.ring_n <= 1) return a.x;
    const int j = ldg_o(&a.sc->k) % a.ring_n;
    return j == 0 ? a.x : a.ring + (int64_t)(j - 1) * a.ring_stride;
}

// Block sums of two values in a fixed order; valid in thread 0.
__device__ __forceinline__ double2 block_reduce2(double u, double v, double *sh /*[64]*/) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    __syncwarp();
    u = warp_sum(u);
    v = warp_sum(v);
    if (lane == 0) {
        sh[warp] = u;
        sh[32 + warp] = v;
    }
    __syncwarp();
    __syncthreads();
    if (warp == 0) {
        u = warp_sum(lane < kWarps ? sh[lane] : 0.0);
        v = warp_sum(lane < kWarps ? sh[32 + lane] : 0.0);
    }
    return make_double2(u, v);
}

// kDots 2 epilogue: per-block (gamma, delta) partials.
__device__ __forceinline__ void spmv_sr_partials(const SpmvArgs &a, double g, double d) {
    __shared__ double sh2[64];
    const double2 t = block_reduce2(g, d, sh2);
    if (threadIdx.x == 0) {
        a.parts_only[a.part_base + spmv_bid(a)] = t.x;
        a.parts_only[a.total_blocks + a.part_base + spmv_bid(a)] = t.y;
    }
}

// kDots: 0 plain y = A x; 1 CG epilogue p.Ap (x = p, y = Ap); 2 the f2
// single-reduction epilogue gamma = x.x and delta = y.x (x = r, y = w = A r),
// both from the diagonal slot's gathered value (no extra bytes), written as
// per-block partials parts_only[b] and parts_only[total_blocks + b].
// kCheck: return at once when the device `done` flag is set (kDots 2: when
// the run flag run_q[sr_q] says the next iteration does not run) -- plain /
// per-iteration-graph launches; the while-graph never launches past
// convergence so it skips that load, whose latency would otherwise sit in
// front of every block's first matrix load).
// kMinB: __launch_bounds__ min blocks per SM (register budget 65536/(256 kMinB)).
template <int kDots, bool kCheck, int kMinB>
__global__ void __launch_bounds__(kBlock, kMinB) spmv27_kernel(SpmvArgs a) {
    int64_t row, lim;
    const int64_t bid = spmv_bid(a);
    if (bid < a.nb0) {
        row = a.r0 + bid * kBlock + threadIdx.x;
        lim = a.r0 + a.len0;
    } else {
        row = a.r1 + (bid - a.nb0) * kBlock + threadIdx.x;
        lim = a.r1 + a.len1;
    }
    constexpr bool kDot = kDots == 1;
    double d = 0.0, dg = 0.0;  // kDots 1: p.Ap; kDots 2: delta (d) and gamma (dg)
    // The first matrix loads are issued before waiting for the predecessor
    // (PDL) and before the done flag is read, so neither latency sits in
    // front of the stream.
    int done = 0;
    if (row < lim) {
        const uint64_t pol = policy_evict_first();
        const double *v = a.val + row;
        const int *c = a.col + row;
        double sum = 0.0;  // FMA chain in ascending column from +0.0 (A8)
        double xd = 0.0;
        int cd = 0;
        const double *xg = a.x;
        // three groups of 9 slots (one z-plane of the stencil each); all 18
        // loads of a group are issued before its gathers and FMAs, and the
        // compiler may hoist the next group's loads above them
#pragma unroll
        for (int g = 0; g < 3; ++g) {
            double vv[9];
            int cc[9];
#pragma unroll
            for (int t = 0; t < 9; ++t) {
                vv[t] = ld_stream(v + (9 * g + t) * a.stride, pol);
                cc[t] = ld_stream(c + (9 * g + t) * a.stride, pol);
            }
            if (g == 0) {
                pdl_wait();
                if (a.early_trigger) pdl_trigger();
                if (kDot && a.trace) trace_mark(a.trace, a.trace_max, ldg_o(&a.sc->k), 1, false);
                done = spmv_done<kDots, kCheck>(a);
                if (done) return;  // uniform over the grid, before any store
                xg = spmv_xg(a);
            }
#pragma unroll
            for (int t = 0; t < 9; ++t) {
                const double xv = __ldg(xg + cc[t]);
                if (9 * g + t == kDiagSlot) {
                    xd = xv;
                    cd = cc[t];
                }
                sum = fma(vv[t], xv, sum);
            }
        }
        a.y[row] = sum;
        // p_i: the diagonal slot's gathered value when that slot really is the
        // row's own column (always, for generated matrices); else reload it.
        if (kDots > 0) {
            const double xi = cd == row + a.plane ? xd : __ldg(xg + row + a.plane);
            d = sum * xi;
            if (kDots == 2) dg = xi * xi;
        }
    } else {
        pdl_wait();
        done = spmv_done<kDots, kCheck>(a);
    }
    pdl_trigger();  // (a second launch_dependents after an early one is a no-op)
    if (done) return;
    if (kDots == 2) {
        spmv_sr_partials(a, dg, d);
        return;
    }
    if (kDot && a.trace) trace_mark(a.trace, a.trace_max, ldg_o(&a.sc->k), 1, true);
    if (kDot) {
        if (a.parts_only) {  // block partial only; the update kernel sums them
            __shared__ double shp[32];
            d = block_reduce<false>(d, shp);
            if (threadIdx.x == 0) a.parts_only[a.part_base + bid] = d;
            return;
        }
        CgScalars *sc = a.sc;
        const int single = a.single;
        grid_reduce<false>(d, a.red, a.part_base + (unsigned)bid, a.total_blocks,
                           [sc, single](double s) {
                               if (single) sc->pAp = s; else sc->loc_pAp = s;
                           });
    }
}

// Two adjacent rows per thread: 16-B `val` and 8-B `col` loads (half the
// load instructions of spmv27_kernel for the same bytes), 9 groups of 3 slots.
// Half as many blocks also halves the per-block cost of the last-block
// finisher (its fence + ticket round trip holds the block's SM slot) --
// measured on B200 at 128^3: 105.8 us vs 108.4 us with the p.Ap epilogue
// (tools/spmvbench.cu).  Needs even n (stride), even range starts and a 16-B
// aligned y (the host checks); a range of odd length ends in a 1-row thread.
// Same per-row FMA order as spmv27_kernel: identical bits.
// HALO_PEER = 2 boundary block: wait until the neighbours whose halo planes
// rows [first, last] read have pushed p of iteration k (uniform per block)
__device__ __forceinline__ void fused_halo_wait(const SpmvArgs &a, int64_t first, int64_t last) {
    if (threadIdx.x == 0) {
        const PeerTab *t = a.fpeer;
        // iteration k's SpMV: niters = k (written by the p update / f2 update)
        const unsigned long long tg = ftag(ldg_o(&a.sc->epoch), (unsigned long long)ldg_o(&a.sc->niters));
        if (first < a.plane && t->rank > 0)
            spin_until(&t->mine->fflag_from_lo, tg, t->mine, PEER_WAIT_HALO_LO, t->rank - 1);
        if (last >= a.stride - a.plane && t->rank < t->nranks - 1)
            spin_until(&t->mine->fflag_from_hi, tg, t->mine, PEER_WAIT_HALO_HI, t->rank + 1);
    }
    __syncthreads();
}

// kFused (HALO_PEER = 2, multi-slab CG SpMV): ranges 1 and 2 are the boundary
// planes; their blocks (the last ones in block order) wait for the halo flags
// before any load (fused_halo_wait) and gather through L2 (ld.global.cg: the
// halo was written by a peer during this grid's lifetime, so the read-only
// path is not allowed for it); interior blocks are unchanged.
template <bool kCoh>
__device__ __forceinline__ double ld_gather(const double *p) {
    return kCoh ? __ldcg(p) : __ldg(p);
}

// kDia (HPCCG_OPT_SPMV_FORMAT = 1, DIA-27 reading of the same ELL): the column
// of slot s is not loaded but formed from the stencil offset the generator
// placed there (gen27_kernel: col = own + sz*plane + sy*nx + sx when the
// neighbour exists, else the padding (0.0, own)); a zero value selects the
// padding column, so every FMA sees the same (val, x) pair as the ELL kernel
// and the result is bitwise identical.  Valid for matrices made by
// hpccg_generate (the only source of matrices in this library): structurally
// present entries are 27 or -1, never 0.  Saves the 4 B/slot index stream:
// 216 B/row of values instead of 324 B/row of values + indices.
#ifndef HPCCG_DIA_GROUP
#define HPCCG_DIA_GROUP 9  // measured: 9 > 3 (27 spills at 64 registers), DESIGN.md sec. 7.1
#endif
constexpr int kDiaGroup = HPCCG_DIA_GROUP;  // 3 or 9
#ifndef HPCCG_DIA_MINB
#define HPCCG_DIA_MINB 4  // resident 256-thread blocks per SM (64 registers)
#endif
constexpr int kDiaMinB = HPCCG_DIA_MINB;
static_assert(kSlots % kDiaGroup == 0, "DIA group must divide 27");

template <bool kDia>
__device__ __forceinline__ int2 spmv_cols(const SpmvArgs &a, const int *c, int s, double2 v, int64_t row,
                                          uint64_t pol) {
    if (!kDia) return ld_stream2(c + s * a.stride, pol);
    const int own = (int)(row + a.plane);
    const int off = (s / 9 - 1) * (int)a.plane + ((s / 3) % 3 - 1) * a.nx + (s % 3 - 1);
    return make_int2(v.x != 0.0 ? own + off : own, v.y != 0.0 ? own + 1 + off : own + 1);
}

// HPCCG_OPT_SPMV_CLUSTER: the single-slab CG SpMV launched in clusters of
// kSpmvCl CTAs; each cluster folds its CTAs' p.Ap partials (row-block order)
// into ONE partial through distributed shared memory, so a 256^3 slab
// leaves 4096 partials -- few enough for every update block to sum itself, no
// 1024-thread finisher kernel between the SpMV and the update
constexpr int kSpmvCl = 8;

template <int kDots, bool kCheck, bool kFused, bool kCoh, bool kDia = false, bool kCl = false, bool kRing = false>
__device__ __forceinline__ void spmv27x2_body(const SpmvArgs &a, int64_t row, int64_t lim, int64_t bid) {
    constexpr bool kDot = kDots == 1;
    double d = 0.0, dg = 0.0;  // kDots 1: p.Ap; kDots 2: delta (d) and gamma (dg)
    int done = 0;
    if (row + 1 < lim) {
        const uint64_t pol = policy_evict_first();
        const double *v = a.val + row;
        const int *c = a.col + row;
        double s0 = 0.0, s1 = 0.0, x0 = 0.0, x1 = 0.0;
        int c0 = 0, c1 = 0;
        // kRing: the slot of sc->k (set after the wait); else the parameter itself
        // (no copy held in a register)
        const double *xgr = nullptr;
#define XG (kRing ? xgr : a.x)
        // slots whose loads are issued together: 3 (ELL: 72 B per thread in
        // flight); DIA has no index stream, so it takes kDiaGroup slots
        constexpr int kG = kDia ? kDiaGroup : 3;
#pragma unroll
        for (int g = 0; g < kSlots / kG; ++g) {
            double2 vv[kG];
            int2 cc[kG];
#pragma unroll
            for (int t = 0; t < kG; ++t) {
                vv[t] = ld_stream2(v + (kG * g + t) * a.stride, pol);
                if (!kDia) cc[t] = ld_stream2(c + (kG * g + t) * a.stride, pol);
            }
            if (g == 0) {
                pdl_wait();
                if (a.early_trigger) pdl_trigger();
                if (kDot && a.trace) trace_mark(a.trace, a.trace_max, ldg_o(&a.sc->k), 1, false);
                done = spmv_done<kDots, kCheck>(a);
                if (done) return;  // uniform over the grid, before any store
                if (kRing) xgr = spmv_xg<true>(a);
            }
#pragma unroll
            for (int t = 0; t < kG; ++t) {
                if (kDia) cc[t] = spmv_cols<true>(a, c, kG * g + t, vv[t], row, pol);
                const double xa = ld_gather<kCoh>(XG + cc[t].x), xb = ld_gather<kCoh>(XG + cc[t].y);
                if (kG * g + t == kDiagSlot) {
                    x0 = xa;
                    x1 = xb;
                    c0 = cc[t].x;
                    c1 = cc[t].y;
                }
                s0 = fma(vv[t].x, xa, s0);
                s1 = fma(vv[t].y, xb, s1);
            }
        }
        if (kDots == 1) st_hint<2>(reinterpret_cast<double2 *>(a.y + row), make_double2(s0, s1));
        else *reinterpret_cast<double2 *>(a.y + row) = make_double2(s0, s1);
        if (kDots > 0) {
            const double p0 = c0 == row + a.plane ? x0 : ld_gather<kCoh>(XG + row + a.plane);
            const double p1 = c1 == row + 1 + a.plane ? x1 : ld_gather<kCoh>(XG + row + 1 + a.plane);
#undef XG
            d = fma(s1, p1, s0 * p0);
            if (kDots == 2) dg = fma(p1, p1, p0 * p0);
        }
    } else if (row < lim) {  // odd tail: one row, scalar loads
        const uint64_t pol = policy_evict_first();
        pdl_wait();
        done = spmv_done<kDots, kCheck>(a);
        if (done) return;
        const double *xg = spmv_xg<kRing>(a);
        double s0 = 0.0;
#pragma unroll
        for (int k = 0; k < kSlots; ++k)
            s0 = fma(ld_stream(a.val + k * a.stride + row, pol),
                     ld_gather<kCoh>(xg + ld_stream(a.col + k * a.stride + row, pol)), s0);
        a.y[row] = s0;
        if (kDots > 0) {
            const double xi = ld_gather<kCoh>(xg + row + a.plane);
            d = s0 * xi;
            if (kDots == 2) dg = xi * xi;
        }
    } else {
        pdl_wait();
        done = spmv_done<kDots, kCheck>(a);
    }
    pdl_trigger();  // (a second launch_dependents after an early one is a no-op)
    if (done) return;
    if (kDots == 2) {
        spmv_sr_partials(a, dg, d);
        return;
    }
    if (kDot && a.trace) trace_mark(a.trace, a.trace_max, ldg_o(&a.sc->k), 1, true);
    if (kDot) {
        if (a.parts_only) {  // block partial only; the update kernel sums them
            __shared__ double shp[32];
            d = block_reduce<false>(d, shp);
            if (kCl) {
                __shared__ double clp[kSpmvCl];
                namespace cgx = cooperative_groups;
                cgx::cluster_group cl = cgx::this_cluster();
                // slot by row block (not cluster rank): the same sum when the grid
                // walks the rows backwards (serpentine)
                if (threadIdx.x == 0) *cl.map_shared_rank(&clp[bid % kSpmvCl], 0) = d;
                cl.sync();
                if (cl.block_rank() == 0 && threadIdx.x == 0) {
                    double t = clp[0];
#pragma unroll
                    for (int c = 1; c < kSpmvCl; ++c) t += clp[c];
                    a.parts_only[a.part_base + bid / kSpmvCl] = t;
                }
                return;
            }
            if (threadIdx.x == 0) a.parts_only[a.part_base + bid] = d;
            return;
        }
        CgScalars *sc = a.sc;
        const int single = a.single;
        const PeerTab *fp = kFused ? a.fpeer : nullptr;
        grid_reduce<false>(d, a.red, a.part_base + (unsigned)bid, a.total_blocks,
                           [sc, single, fp](double s) {
                               if (single) sc->pAp = s; else sc->loc_pAp = s;
                               if (kFused)  // p.Ap(k) -> slot 1 of every rank
                                   fused_post(fp, 1, s, ll_tag(sc->epoch, 2ull * (unsigned)sc->k - 1ull));
                           });
    }
}


// Single slab, p.Ap partials for the finisher-free update (HPCCG_OPT_SPMV_TRIPS):
// each block SpMVs `trips` consecutive 512-row trips (range 0 only) and writes
// ONE partial, so a large slab (256^3: 32768 row blocks) leaves <= 4096
// partials, which every update block sums itself -- no 1024-thread p.Ap
// finisher kernel between the SpMV and the update.  Per row the same FMA chain
// as spmv27x2_kernel (identical Ap bits); the partial tree differs (the sum
// goes trip by trip per thread, then the block).
template <bool kCheck>
__global__ void __launch_bounds__(kBlock, 4) spmv27x2_trips_kernel(SpmvArgs a) {
    const int64_t bid = spmv_bid(a);
    const int64_t lim = a.r0 + a.len0;
    const uint64_t pol = policy_evict_first();
    double d = 0.0;
    for (int t = 0; t < a.trips; ++t) {
        const int64_t row = a.r0 + ((bid * a.trips + t) * kBlock + threadIdx.x) * 2;
        if (row >= lim) {
            if (t == 0) {
                pdl_wait();
                if (spmv_done<1, kCheck>(a)) return;
            }
            break;
        }
        if (row + 1 < lim) {
            const double *v = a.val + row;
            const int *c = a.col + row;
            double s0 = 0.0, s1 = 0.0, x0 = 0.0, x1 = 0.0;
            int c0 = 0, c1 = 0;
#pragma unroll
            for (int g = 0; g < kSlots / 3; ++g) {
                double2 vv[3];
                int2 cc[3];
#pragma unroll
                for (int u = 0; u < 3; ++u) {
                    vv[u] = ld_stream2(v + (3 * g + u) * a.stride, pol);
                    cc[u] = ld_stream2(c + (3 * g + u) * a.stride, pol);
                }
                if (t == 0 && g == 0) {
                    pdl_wait();
                    if (a.early_trigger) pdl_trigger();
                    if (a.trace) trace_mark(a.trace, a.trace_max, ldg_o(&a.sc->k), 1, false);
                    if (spmv_done<1, kCheck>(a)) return;  // uniform, before any store
                }
#pragma unroll
                for (int u = 0; u < 3; ++u) {
                    const double xa = __ldg(a.x + cc[u].x), xb = __ldg(a.x + cc[u].y);
                    if (3 * g + u == kDiagSlot) {
                        x0 = xa;
                        x1 = xb;
                        c0 = cc[u].x;
                        c1 = cc[u].y;
                    }
                    s0 = fma(vv[u].x, xa, s0);
                    s1 = fma(vv[u].y, xb, s1);
                }
            }
            *reinterpret_cast<double2 *>(a.y + row) = make_double2(s0, s1);
            const double p0 = c0 == row + a.plane ? x0 : __ldg(a.x + row + a.plane);
            const double p1 = c1 == row + 1 + a.plane ? x1 : __ldg(a.x + row + 1 + a.plane);
            d = fma(s1, p1, fma(s0, p0, d));
        } else {  // odd tail: one row
            if (t == 0) {
                pdl_wait();
                if (spmv_done<1, kCheck>(a)) return;
            }
            double s0 = 0.0;
#pragma unroll
            for (int k = 0; k < kSlots; ++k)
                s0 = fma(ld_stream(a.val + k * a.stride + row, pol),
                         __ldg(a.x + ld_stream(a.col + k * a.stride + row, pol)), s0);
            a.y[row] = s0;
            d = fma(s0, __ldg(a.x + row + a.plane), d);
        }
    }
    pdl_trigger();
    if (a.trace) trace_mark(a.trace, a.trace_max, ldg_o(&a.sc->k), 1, true);
    __shared__ double shp[32];
    d = block_reduce<false>(d, shp);
    if (threadIdx.x == 0) a.parts_only[a.part_base + bid] = d;
}

// ---- a.3 + a.4 with the matrix stream fed by TMA (HPCCG_OPT_SPMV_SLICED):
// the CG loop's SpMV reads a CHUNK-SLICED copy of the same ELL-27 matrix --
// chunk c of kSlR rows stored contiguously as val[27][kSlR] doubles followed by
// col[27][kSlR] ints (324 B per row, built once from the slot-major arrays by
// ell_to_sliced_kernel) -- so a whole chunk is ONE cp.async.bulk copy (41.5 KB)
// into a two-stage shared-memory ring per CTA (mbarrier completion).  Persistent
// CTAs (two per SM) take chunks c = b, b + G, ... (reversed under serpentine);
// one row per thread, its 27 column indices and values read from shared memory
// and its 27 gathers of p in flight at once.  The same per-row FMA chain in
// ascending slot order as every other SpMV (identical Ap bits); each thread
// accumulates its p.Ap over its chunks in order and each CTA writes ONE partial,
// so the update sums G <= 4096 partials itself -- no p.Ap finisher kernel.
// Measured at 256^3 (tools/tmaspmv.cu): 792 vs 802 us per SpMV (7.15 TB/s on
// 12 nnz + 16n B); a TMA copy per slot of the slot-major arrays instead (54 per
// chunk) is issue-bound at 2.6-3.8 TB/s.  In the CG loop the gain depends on
// the box (DESIGN 7.1): opt-in.
constexpr int kSlR = 128;                  // rows per chunk = threads per CTA
constexpr int kSlStages = 2;
constexpr unsigned kSlBytes = kSlR * 324;  // one chunk: 27 x (8 + 4) B per row

// one thread per row of the padded chunk grid; rows >= n are padding (0.0, the
// halo'd index of row 0's own entry -- a finite value, multiplied by 0)
__global__ void __launch_bounds__(kBlock) ell_to_sliced_kernel(int64_t n, int64_t plane, const double *val,
                                                               const int *col, unsigned char *sl) {
    const int64_t i = (int64_t)blockIdx.x * kBlock + threadIdx.x;
    const int64_t nch = (n + kSlR - 1) / kSlR;
    if (i >= nch * kSlR) return;
    const int64_t c = i / kSlR, j = i % kSlR;
    double *v = reinterpret_cast<double *>(sl + (size_t)c * kSlBytes);
    int *cc = reinterpret_cast<int *>(sl + (size_t)c * kSlBytes + (size_t)kSlR * kSlots * 8);
    for (int k = 0; k < kSlots; ++k) {
        v[k * kSlR + j] = i < n ? val[(int64_t)k * n + i] : 0.0;
        cc[k * kSlR + j] = i < n ? col[(int64_t)k * n + i] : (int)plane;
    }
}

// one chunk into a stage; the matrix is read once per SpMV: evict-first in L2,
// so it does not push out the planes of p the gathers reuse
// (measured without the hint: 512^3 8496 vs 7880 us/iteration -- the stream
// evicted the gathered planes of p)
__device__ __forceinline__ void sl_issue(const unsigned char *src, unsigned char *dst, unsigned long long *bar) {
    const unsigned mb = (unsigned)__cvta_generic_to_shared(bar);
    const uint64_t pol = policy_evict_first();
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(kSlBytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
                 ::"r"((unsigned)__cvta_generic_to_shared(dst)), "l"(src), "r"(kSlBytes), "r"(mb), "l"(pol) : "memory");
}

__device__ __forceinline__ void sl_wait(unsigned long long *bar, unsigned parity) {
    const unsigned mb = (unsigned)__cvta_generic_to_shared(bar);
    unsigned ok = 0;
    while (!ok)
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                     : "=r"(ok) : "r"(mb), "r"(parity) : "memory");
}

template <bool kCheck>
__global__ void __launch_bounds__(kSlR, 2) spmv_sliced_kernel(SpmvArgs a, const unsigned char *sl) {
    extern __shared__ __align__(128) unsigned char ring[];
    __shared__ __align__(8) unsigned long long full[kSlStages];
    __shared__ double shp[32];
    const int64_t n = a.len0, nch = (n + kSlR - 1) / kSlR;
    const int64_t G = gridDim.x, b = blockIdx.x;
    const int64_t mine = b < nch ? (nch - 1 - b) / G + 1 : 0;
    auto chunk = [&](int64_t i) { const int64_t c = b + i * G; return a.rev ? nch - 1 - c : c; };
    // the matrix does not depend on the predecessor: the first stages are in
    // flight before the PDL wait
    if (threadIdx.x == 0) {
        for (int s = 0; s < kSlStages; ++s)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((unsigned)__cvta_generic_to_shared(&full[s])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int s = 0; s < kSlStages && s < mine; ++s)
            sl_issue(sl + (size_t)chunk(s) * kSlBytes, ring + (size_t)s * kSlBytes, &full[s]);
    }
    __syncthreads();
    pdl_wait();
    if (a.early_trigger) pdl_trigger();
    if (a.trace) trace_mark(a.trace, a.trace_max, ldg_o(&a.sc->k), 1, false);
    if (spmv_done<1, kCheck>(a)) {  // uniform: let the copies in flight land before leaving
        for (int s = 0; s < kSlStages && s < mine; ++s) sl_wait(&full[s], 0);
        return;
    }
    const double *xg = spmv_xg<true>(a);  // p's ring slot (ring-deferred x update) or a.x
    double d = 0.0;
    for (int64_t i = 0; i < mine; ++i) {
        const int s = (int)(i % kSlStages);
        sl_wait(&full[s], (unsigned)((i / kSlStages) & 1));
        const unsigned char *st = ring + (size_t)s * kSlBytes;
        const double *sv = reinterpret_cast<const double *>(st);
        const int *sc = reinterpret_cast<const int *>(st + (size_t)kSlR * kSlots * 8);
        const int j = threadIdx.x;
        const int64_t row = chunk(i) * kSlR + j;
        double xv[kSlots];
        int cd = 0;
#pragma unroll
        for (int k = 0; k < kSlots; ++k) {  // all 27 gathers in flight
            const int cc = sc[k * kSlR + j];
            if (k == kDiagSlot) cd = cc;
            xv[k] = __ldg(xg + cc);
        }
        double s0 = 0.0;  // FMA chain in ascending column from +0.0 (A8)
#pragma unroll
        for (int k = 0; k < kSlots; ++k) s0 = fma(sv[k * kSlR + j], xv[k], s0);
        __syncthreads();  // stage s consumed by every thread
        if (threadIdx.x == 0 && i + kSlStages < mine)
            sl_issue(sl + (size_t)chunk(i + kSlStages) * kSlBytes, ring + (size_t)s * kSlBytes, &full[s]);
        if (row < n) {
            a.y[row] = s0;
            const double p0 = cd == row + a.plane ? xv[kDiagSlot] : __ldg(xg + row + a.plane);
            d = fma(s0, p0, d);
        }
    }
    pdl_trigger();
    if (a.trace) trace_mark(a.trace, a.trace_max, ldg_o(&a.sc->k), 1, true);
    // CTA sum of kSlR / 32 warps (block_reduce assumes kBlock threads)
    d = warp_sum(d);
    if ((threadIdx.x & 31) == 0) shp[threadIdx.x >> 5] = d;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = shp[0];
#pragma unroll
        for (int w = 1; w < kSlR / 32; ++w) t += shp[w];
        a.parts_only[a.part_base + b] = t;
    }
}

// (the fused z-slab kernel with the ring slot pointer: 3 blocks per SM -- at
// 64 registers its kCheck variant spills, 849 vs 813 us at 256^3)
template <int kDots, bool kCheck, bool kFused = false, bool kDia = false, bool kRing = false>
__global__ void __launch_bounds__(kBlock, kDia ? kDiaMinB : (kFused && kRing ? 3 : 4)) spmv27x2_kernel(SpmvArgs a) {
    int64_t row, lim;
    const int64_t bid = spmv_bid(a);
    bool bnd = false;
    if (bid < a.nb0) {
        row = a.r0 + (bid * kBlock + threadIdx.x) * 2;
        lim = a.r0 + a.len0;
    } else if (!kFused || bid < a.nb01) {
        row = a.r1 + ((bid - a.nb0) * kBlock + threadIdx.x) * 2;
        lim = a.r1 + a.len1;
        bnd = kFused;
    } else {
        row = a.r2 + ((bid - a.nb01) * kBlock + threadIdx.x) * 2;
        lim = a.r2 + a.len2;
        bnd = true;
    }
    if (kFused && bnd) {
        // only blocks that read a halo some neighbour fills wait (and load
        // coherently); `done` first: past convergence nobody pushes
        const int64_t first = row - 2 * (int64_t)threadIdx.x, last = min(first + 2 * kBlock, lim) - 1;
        const PeerTab *t = a.fpeer;
        bnd = (first < a.plane && t->rank > 0) || (last >= a.stride - a.plane && t->rank < t->nranks - 1);
        if (bnd) {
            // niters / done are written by the predecessor (PDL): wait for it
            // first (the body's second griddepcontrol.wait is a no-op)
            pdl_wait();
            if (kCheck && ldg_o(&a.sc->done)) return;  // uniform exit
            fused_halo_wait(a, first, last);
        }
    }
    if (kFused && bnd) {
        spmv27x2_body<kDots, kCheck, kFused, true, kDia, false, kRing>(a, row, lim, bid);
        return;
    }
    spmv27x2_body<kDots, kCheck, kFused, false, kDia, false, kRing>(a, row, lim, bid);
}

// the single-slab CG SpMV in clusters of kSpmvCl CTAs (grid a multiple of
// kSpmvCl; the padding blocks have no rows and contribute 0)
template <bool kCheck, bool kRing>
__global__ void __launch_bounds__(kBlock, 4) spmv27x2_cl_kernel(SpmvArgs a) {
    const int64_t bid = spmv_bid(a);
    const int64_t row = a.r0 + (bid * kBlock + threadIdx.x) * 2, lim = a.r0 + a.len0;
    spmv27x2_body<1, kCheck, false, false, false, true, kRing>(a, row, lim, bid);
}

// ------------------------------------------------ streaming vector kernels
// Device scalars are read with weak L1-cacheable loads after the PDL wait
// (ldg_o): one L2 request per SM serves every warp.  (Volatile reads from
// every warp all hit the one L2 slice that owns the scalar line and serialise
// there -- measured: 2x slower vector kernels; and the read-only path may be
// hoisted above the wait, see ldg_o.)
// Grids walk the vectors in 16-B double2 units, one unit per thread per trip;
// by default one thread per unit (a full, non-persistent grid: 2048 resident
// threads per SM keep enough loads in flight), or a persistent grid of
// HPCCG_OPT_VEC_WAVES waves (SM count x resident blocks).  Scalar (8-B) path when a pointer is not 16-B aligned.  The
// element -> thread mapping depends only on (n, grid): reductions are
// run-to-run deterministic.

__device__ __forceinline__ int64_t gtid() { return (int64_t)blockIdx.x * kBlock + threadIdx.x; }
__device__ __forceinline__ int64_t gnth() { return (int64_t)gridDim.x * kBlock; }

// a.6: p = r + beta p  (k == 1: p = r)            -- 24n B
// kU: 16-B units per thread per trip, all loads issued before any store
// (memory-level parallelism for DRAM-resident vectors).  The per-thread
// element order is the same for every kU, so kU never changes the bits.
template <bool kVec, bool kCheck, int kU>
__global__ void __launch_bounds__(kBlock) cg_pupdate_kernel(int64_t n, const double *__restrict__ r,
                                                           double *__restrict__ p,
                                                           const CgScalars *sc, TraceSlot *trace,
                                                           int trace_max) {
    pdl_wait();
    pdl_trigger();
    const int ktr = trace ? ldg_o(&sc->k) : 0;
    trace_mark(trace, trace_max, ktr, 0, false);
    // `done` is tested after each trip's loads (never in front of them)
    const int done = kCheck ? ldg_o(&sc->done) : 0;
    const bool first = (ldg_o(&sc->k) == 1);
    const double beta = first ? 0.0 : ldg_o(&sc->rr_cur) / ldg_o(&sc->rr_prev);
    const int64_t tid = gtid(), nth = gnth();
    if (kVec) {
        const int64_t nv = n >> 1;
        const double2 *__restrict__ r2 = reinterpret_cast<const double2 *>(r);
        double2 *__restrict__ p2 = reinterpret_cast<double2 *>(p);
        for (int64_t b = tid; b < nv; b += kU * nth) {
            double2 ra[kU], pa[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int64_t i = b + u * nth;
                if (i < nv) {
                    ra[u] = r2[i];
                    pa[u] = p2[i];
                }
            }
            if (done) return;
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int64_t i = b + u * nth;
                if (i < nv) {
                    double2 q = ra[u];
                    if (!first) {
                        q.x = fma(beta, pa[u].x, ra[u].x);
                        q.y = fma(beta, pa[u].y, ra[u].y);
                    }
                    p2[i] = q;
                }
            }
        }
        if (done) return;
        if (tid == 0 && (n & 1)) {
            const int64_t i = n - 1;
            p[i] = first ? r[i] : fma(beta, p[i], r[i]);
        }
    } else {
        if (done) return;
        for (int64_t i = tid; i < n; i += nth) p[i] = first ? r[i] : fma(beta, p[i], r[i]);
    }
    if (trace) {
        __syncthreads();  // the block's stores are issued before its end mark
        trace_mark(trace, trace_max, ktr, 0, true);
    }
}

// a.5: x += alpha p; r -= alpha Ap; partial r.r; then the loop control of
// the NEXT iteration (A4 lagged check, A11 guard) in the last block, which
// also drives the while-graph's condition (`cond`, 0 = none).  48n B.
struct UpdArgs {
    int64_t n;
    double *x, *r;
    const double *p, *Ap;
    const double *pAp_parts;  // non-null: p.Ap = fixed-order sum of these
    unsigned n_parts;
    TraceSlot *trace;
    int trace_max;
    CgScalars *sc;
    Reduction red;
    int single;
    unsigned long long cond;  // cudaGraphConditionalHandle or 0
};

__device__ __forceinline__ void set_cond(unsigned long long h, int cont) {
    if (h) cudaGraphSetConditional((cudaGraphConditionalHandle)h, cont ? 1u : 0u);
}

// p.Ap from the SpMV's block partials when there are too many for every
// update block to sum them (> kUpdSumMax): one 1024-thread block, fixed order.
constexpr unsigned kUpdSumMax = 4096;

// The same sum over kPapCl CTAs of one thread-block cluster: CTA c reduces the
// c-th contiguous share of the partials (8 independent loads in flight per
// thread), the leader adds the kPapCl CTA sums in rank order from distributed
// shared memory.  32768 partials (256^3) are 256 KB: one SM's L2 bandwidth and
// latency set the single-CTA finisher's ~5.3 us; eight SMs read them in
// parallel.  Deterministic (fixed shares and order), another tree than
// cg_pap_finish_kernel's.
constexpr int kPapCl = 8;
__global__ void __launch_bounds__(1024, 1) cg_pap_finish_cl_kernel(const double *parts, unsigned n_parts,
                                                                CgScalars *sc) {
    namespace cgx = cooperative_groups;
    pdl_wait();
    pdl_trigger();
    __shared__ double sh[32];
    __shared__ double s_res;
    auto cl = cgx::this_cluster();
    const unsigned rank = cl.block_rank();
    const unsigned share = (n_parts + kPapCl - 1) / kPapCl;
    const unsigned lo = rank * share, hi = min(n_parts, lo + share);
    double acc[8] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
    unsigned i = lo + threadIdx.x;
    for (; i + 7u * 1024u < hi; i += 8u * 1024u) {
        double v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = ldg_o(parts + i + u * 1024u);
#pragma unroll
        for (int u = 0; u < 8; ++u) acc[u] += v[u];
    }
    for (; i < hi; i += 1024) acc[0] += ldg_o(parts + i);
    double q = ((acc[0] + acc[1]) + (acc[2] + acc[3])) + ((acc[4] + acc[5]) + (acc[6] + acc[7]));
    q = warp_sum(q);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = q;
    __syncthreads();
    if (threadIdx.x < 32) {
        q = warp_sum(sh[threadIdx.x]);
        if (threadIdx.x == 0) s_res = q;
    }
    cl.sync();
    if (rank == 0 && threadIdx.x == 0) {
        double t = 0.0;
        for (int c = 0; c < kPapCl; ++c) t += *cl.map_shared_rank(&s_res, c);
        sc->pAp = t;
    }
    cl.sync();  // the leader has read every CTA's s_res before any CTA exits
}

__global__ void __launch_bounds__(1024, 1) cg_pap_finish_kernel(const double *parts, unsigned n_parts,
                                                             CgScalars *sc) {
    pdl_wait();
    pdl_trigger();
    __shared__ double sh[32];
    // 8 independent loads in flight per thread (32768 partials at 256^3:
    // one L2 round trip per 8 instead of a dependent chain of 32)
    double acc[8] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
    unsigned i = threadIdx.x;
    // 3 trips' loads (24) in flight, then added trip by trip: the same order as
    // the 8-wide loop below, so the same bits (262144 partials at 512^3).  The
    // partials come from the previous grid (complete after pdl_wait), so the
    // read-only path is valid -- and lets ptxas issue the whole batch at once
    // (ld.cg loads were interleaved with the adds, ~4 in flight)
    for (; i + 23u * 1024u < n_parts; i += 24u * 1024u) {
        double v[24];
#pragma unroll
        for (int u = 0; u < 24; ++u) v[u] = ldg_o(parts + i + u * 1024u);
#pragma unroll
        for (int t = 0; t < 3; ++t)
#pragma unroll
            for (int u = 0; u < 8; ++u) acc[u] += v[8 * t + u];
    }
    for (; i + 7u * 1024u < n_parts; i += 8u * 1024u) {
#pragma unroll
        for (int u = 0; u < 8; ++u) acc[u] += __ldcg(parts + i + u * 1024u);
    }
    for (; i < n_parts; i += 1024) acc[0] += __ldcg(parts + i);
    double q = ((acc[0] + acc[1]) + (acc[2] + acc[3])) + ((acc[4] + acc[5]) + (acc[6] + acc[7]));
    q = warp_sum(q);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = q;
    __syncthreads();
    if (threadIdx.x < 32) {
        q = warp_sum(sh[threadIdx.x]);
        if (threadIdx.x == 0) sc->pAp = q;
    }
}

template <bool kVec, bool kCheck, int kU>
__global__ void __launch_bounds__(kBlock) cg_update_kernel(UpdArgs a) {
    CgScalars *sc = a.sc;
    pdl_wait();
    pdl_trigger();
    const int ktr = a.trace ? ldg_o(&sc->k) : 0;
    trace_mark(a.trace, a.trace_max, ktr, 2, false);
    // `done` is tested after each trip's loads (never in front of them); it
    // is uniform over the grid, so every block leaves before the reduction.
    const int done = kCheck ? ldg_o(&sc->done) : 0;
    const double rtrans = ldg_o(&sc->rr_cur);
    double pAp;
    if (a.pAp_parts) {
        // every block sums the SpMV's partials in the same fixed order, so
        // every block holds the bit-identical p.Ap (no grid-wide finisher)
        __shared__ double shq[32];
        double q = 0.0;
        for (unsigned i = threadIdx.x; i < a.n_parts; i += kBlock) q += __ldcg(a.pAp_parts + i);
        q = block_reduce<false>(q, shq);
        if (threadIdx.x == 0) shq[31] = q;
        __syncthreads();
        pAp = shq[31];
    } else {
        pAp = ldg_o(&sc->pAp);
    }
    const bool stop = (rtrans == 0.0) || (pAp == 0.0);  // A11
    const double alpha = stop ? 0.0 : rtrans / pAp;
    const int64_t tid = gtid(), nth = gnth();
    double acc = 0.0, acc2 = 0.0;
    if (kVec) {
        const int64_t nv = a.n >> 1;
        double2 *__restrict__ x2 = reinterpret_cast<double2 *>(a.x);
        double2 *__restrict__ r2 = reinterpret_cast<double2 *>(a.r);
        const double2 *__restrict__ p2 = reinterpret_cast<const double2 *>(a.p);
        const double2 *__restrict__ q2 = reinterpret_cast<const double2 *>(a.Ap);
        for (int64_t b = tid; b < nv; b += kU * nth) {
            double2 xa[kU], ra[kU], pa[kU], qa[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int64_t i = b + u * nth;
                if (i < nv) {
                    xa[u] = x2[i];
                    ra[u] = r2[i];
                    pa[u] = p2[i];
                    qa[u] = q2[i];
                }
            }
            if (done) return;
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int64_t i = b + u * nth;
                if (i < nv) {
                    xa[u].x = fma(alpha, pa[u].x, xa[u].x);
                    xa[u].y = fma(alpha, pa[u].y, xa[u].y);
                    ra[u].x = fma(-alpha, qa[u].x, ra[u].x);
                    ra[u].y = fma(-alpha, qa[u].y, ra[u].y);
                    x2[i] = xa[u];
                    r2[i] = ra[u];
                    acc = fma(ra[u].x, ra[u].x, acc);
                    acc2 = fma(ra[u].y, ra[u].y, acc2);
                }
            }
        }
        if (done) return;
        if (tid == 0 && (a.n & 1)) {
            const int64_t i = a.n - 1;
            a.x[i] = fma(alpha, a.p[i], a.x[i]);
            const double rv = fma(-alpha, a.Ap[i], a.r[i]);
            a.r[i] = rv;
            acc = fma(rv, rv, acc);
        }
        acc += acc2;
    } else {
        if (done) return;
        for (int64_t i = tid; i < a.n; i += nth) {
            a.x[i] = fma(alpha, a.p[i], a.x[i]);
            const double rv = fma(-alpha, a.Ap[i], a.r[i]);
            a.r[i] = rv;
            acc = fma(rv, rv, acc);
        }
    }
    const int single = a.single;
    const unsigned long long cond = a.cond;
    trace_mark(a.trace, a.trace_max, ktr, 2, true);
    grid_reduce<false>(acc, a.red, blockIdx.x, gridDim.x,
                       [sc, single, rtrans, stop, cond, pAp](double s) {
                           sc->pAp = pAp;
                           sc->rr_prev = rtrans;
                           if (single) sc->rr_cur = s; else sc->loc_rr = s;
                           const int k = sc->k;
                           const double normr = sqrt(rtrans);
                           sc->normr = normr;
                           sc->niters = k;
                           sc->k = k + 1;
                           const int done = stop || !((k + 1) < sc->max_iter && normr > sc->tol);
                           sc->done = done;
                           set_cond(cond, !done);
                       });
}

// ------------------- single slab: HPCCG's loop without any grid finisher
// The last-block finisher of cg_update_kernel (fence + atomic ticket + the
// final sum, then the loop control) sits between every update and the next
// p update (~5 us of the 128^3 iteration, DESIGN.md 7.1 trace).  On a single
// slab the reduction can be finished by the CONSUMER instead, as the SpMV's
// p.Ap already is: the update writes its per-block r.r partials, and every
// block of the next p update sums them in the same fixed order as the
// finisher did (identical bits).  The loop decision for iteration k + 1
// (A4: normr = ||r_(k-1)|| lagged, A11: p.Ap) is known inside update k, so
// block 0 of update k takes it.  Device loop state per kernel:
//   p update k  (block 0) writes rr_cur = rtrans_k, normr, niters = k
//   update k    (block 0) writes rr_prev = rtrans_k, pAp, k = k + 1, done,
//               run_q[q] = "iteration k + 1 runs", the while-graph condition
// and every kernel of iteration k reads only what earlier kernels wrote; the
// run flag is double-buffered by iteration parity q = k & 1 (a launch's
// parity is baked into the graph node), so no block reads a word another
// block of its own grid writes.

// HALO_PEER = 2: after a block's halo stores -- the blocks that pushed fence
// (system scope) and take a ticket; the last of the n_push raises the
// neighbours' flags to tg
__device__ __forceinline__ void fused_push_signal(const PeerTab *t, int pushed, unsigned n_push,
                                                  unsigned long long tg) {
    __shared__ int last;
    if (!__syncthreads_or(pushed)) return;
    if (threadIdx.x == 0) {
        __threadfence_system();  // this block's pushes before its ticket
        const unsigned tk = atomicAdd(&t->mine->fpush_ticket, 1u);
        last = (tk == n_push - 1);
    }
    __syncthreads();
    if (!last || threadIdx.x != 0) return;
    __threadfence_system();
    t->mine->fpush_ticket = 0u;
    if (t->lo) st_release_sys(&t->lo->fflag_from_hi, tg);
    if (t->hi) st_release_sys(&t->hi->fflag_from_lo, tg);
}

struct Pupd1Args {
    int64_t n;
    const double *r;
    double *p;
    const double *rr_parts;  // r.r partials of the previous update
    unsigned n_rr;
    const CgScalars *sc_in;
    CgScalars *sc;
    int q;
    TraceSlot *trace;
    int trace_max;
    int rev;  // 1: each thread walks its trips last to first (no reduction: same bits)
    // HALO_PEER = 2 on z-slabs (nullptr: single slab): r.r(k-1) = the P slabs'
    // local sums (block 0 posts this slab's), and the p planes pushed into the
    // neighbours' halos by the n_push blocks that hold boundary rows
    const PeerTab *t;
    int64_t plane;
    unsigned n_push;
    int post;  // 0: the slab's sum was posted by fused_post_kernel (loopback)
    double *x;  // deferred x update (nullptr: off): x += alpha_(k-1) p_(k-1) before p is replaced
};

// Fixed-order sum of n partials (the order of grid_reduce's last block);
// identical in every block.
__device__ __forceinline__ double sum_parts_fixed(const double *parts, unsigned n, double *sh) {
    // the same left-to-right order per thread as the finisher, with 8 loads
    // in flight per batch instead of a dependent chain
    double s = 0.0;
    unsigned i = threadIdx.x;
    for (; i + 7u * kBlock < n; i += 8u * kBlock) {
        double v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = ldg_o(parts + i + u * kBlock);
#pragma unroll
        for (int u = 0; u < 8; ++u) s += v[u];
    }
    for (; i < n; i += kBlock) s += ldg_o(parts + i);
    s = block_reduce<false>(s, sh);
    if (threadIdx.x == 0) sh[32] = s;
    __syncthreads();
    return sh[32];
}

// iteration k does not run: propagate to parity q (block 0), uniform exit
__device__ __forceinline__ bool run_check(CgScalars *sc, int q) {
    if (ldg_o(&sc->run_q[q ^ 1])) return true;
    if (blockIdx.x == 0 && threadIdx.x == 0) sc->run_q[q] = 0;
    return false;
}

// a.6 p = r + beta p for a single slab (HPCCG's k > 1 branch: rtrans = r.r,
// beta = rtrans / oldrtrans; k == 1: p = r).  The first trip's loads are
// issued before the scalar work so their latency overlaps the partial sums.
// kPeer: the HALO_PEER = 2 hooks (z-slabs); the single-slab instantiation
// carries none of their code
// (__launch_bounds__(kBlock, 4) -- 64 registers with spills -- measured slower
// at 256^3: 992 vs 986 us/iteration)
template <int kU, bool kPeer = false>
__global__ void __launch_bounds__(kBlock) cg_pupdate1_kernel(Pupd1Args a) {
    __shared__ double sh[33];
    CgScalars *sc = a.sc;
    const int64_t tid = gtid(), nth = gnth(), nv = a.n >> 1;
    const double2 *__restrict__ r2 = reinterpret_cast<const double2 *>(a.r);
    double2 *__restrict__ p2 = reinterpret_cast<double2 *>(a.p);
    double2 *__restrict__ x2 = reinterpret_cast<double2 *>(a.x);
    double2 ra[kU], pa[kU], xa[kU];
    // deferred x update (HPCCG_OPT_DEFER_X): iteration k > 1 also applies
    // x += alpha_(k-1) p_(k-1) -- the x/r update of iteration k - 1 then moves
    // only r and Ap (24n instead of 48n B) and this pass 40n instead of 24n:
    // 8n B less per iteration, the same FMA on the same operands (same bits)
    const bool dx = a.x != nullptr;
    auto load_p = [&](int64_t b) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < nv) {
                pa[u] = p2[i];
                if (dx) xa[u] = x2[i];
            }
        }
    };
    auto load_r = [&](int64_t b) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < nv) ra[u] = r2[i];
        }
    };
    auto load = [&](int64_t b) {
        load_r(b);
        load_p(b);
    };
    // HPCCG_OPT_SERPENTINE: walking the rows backwards starts where the x/r
    // update (forwards) ended, so the first trips find r and p in L2
    const int64_t step = kU * nth;
    const int64_t b0 = (a.rev && tid < nv) ? tid + ((nv - 1 - tid) / step) * step : tid;
    // p (this kernel's own output one iteration ago) is complete before the
    // update's blocks pass their wait: read it during the update's tail (x
    // too: with the deferred update only this kernel and the init write it)
    load_p(b0);
    pdl_wait();
    pdl_trigger();
    load_r(b0);
    if (!run_check(sc, a.q)) return;
    const int k = ldg_o(&sc->k);
    trace_mark(a.trace, a.trace_max, k, 0, false);
    const bool first = (k == 1);
    const bool upx = dx && !first;
    const double alpha_x = upx ? ldg_o(&sc->alpha_x) : 0.0;
    double rtrans = first ? ldg_o(&sc->rr_cur) : sum_parts_fixed(a.rr_parts, a.n_rr, sh);
    if (kPeer && !first) {  // z-slabs: the slab's r.r -> every rank; the global sum back
        const unsigned tag = ll_tag(ldg_o(&sc->epoch), 2ull * (unsigned)(k - 1));
        if (a.post && blockIdx.x == 0 && threadIdx.x == 0) fused_post(a.t, 0, rtrans, tag);
        rtrans = fused_collect_block(a.t, 0, tag, rtrans, &sh[32]);
    }
    const double beta = first ? 0.0 : rtrans / ldg_o(&sc->rr_prev);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (!first) sc->rr_cur = rtrans;
        sc->normr = sqrt(rtrans);
        sc->niters = k;
    }
    const int64_t n = a.n, plane = a.plane;
    double *lo = kPeer ? a.t->halo_to_lo : nullptr, *hi = kPeer ? a.t->halo_to_hi : nullptr;
    int pushed = 0;
    auto put = [&](int64_t i, double v) {  // row i of the new p -> a neighbour's halo
        if (lo && i < plane) {
            lo[i] = v;
            pushed = 1;
        }
        if (hi && i >= n - plane) {
            hi[i - (n - plane)] = v;
            pushed = 1;
        }
    };
    for (int64_t b = b0; b >= 0 && b < nv;) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < nv) {
                double2 v = ra[u];
                if (!first) {
                    v.x = fma(beta, pa[u].x, ra[u].x);
                    v.y = fma(beta, pa[u].y, ra[u].y);
                }
                if (upx) {
                    xa[u].x = fma(alpha_x, pa[u].x, xa[u].x);
                    xa[u].y = fma(alpha_x, pa[u].y, xa[u].y);
                    x2[i] = xa[u];
                }
                p2[i] = v;
                if (kPeer && (2 * i < plane || 2 * i + 1 >= n - plane)) {
                    put(2 * i, v.x);
                    put(2 * i + 1, v.y);
                }
            }
        }
        b += a.rev ? -step : step;
        if (b >= 0 && b < nv) load(b);
    }
    if (tid == 0 && (n & 1)) {
        const int64_t i = n - 1;
        const double v = first ? a.r[i] : fma(beta, a.p[i], a.r[i]);
        if (upx) a.x[i] = fma(alpha_x, a.p[i], a.x[i]);
        a.p[i] = v;
        if (kPeer) put(i, v);
    }
    if (a.trace) {
        __syncthreads();
        trace_mark(a.trace, a.trace_max, k, 0, true);
    }
    if (kPeer) fused_push_signal(a.t, pushed, a.n_push, ftag(ldg_o(&sc->epoch), (unsigned long long)k));
}

// a.5 x += alpha p, r -= alpha Ap, per-block r.r partial (no finisher), and
// the loop decision for iteration k + 1 (block 0).
struct Upd1Args {
    int64_t n;
    double *x, *r;
    const double *p, *Ap;
    const double *pAp_parts;  // the SpMV's p.Ap partials (nullptr: sc->pAp)
    unsigned n_parts;
    double *rr_parts;         // out: gridDim.x r.r partials
    CgScalars *sc;
    int q;
    unsigned long long cond;
    TraceSlot *trace;
    int trace_max;
    const PeerTab *t;  // HALO_PEER = 2 on z-slabs: p.Ap = the P slabs' local sums
    int post;          // 0: posted by fused_post_kernel (loopback)
    int defer_x;       // 1: leave x to the next p update / cg_xfix_kernel (alpha -> sc->alpha_x)
};
// (kLateP: p was written by the kernel right before -- cg_pspmv_kernel -- so x
// and p are read only after the PDL wait)

// Loopback + HALO_PEER = 2: every slab's kernels share one stream, so a
// collect in slab 0's kernel could never see slab 1's post from a kernel
// queued behind it.  This one-block kernel posts a slab's local sum (its
// partials in the consumers' fixed order, or *fallback) ahead of all the
// consumers.  q 0: r.r(k-1) before p update k (k = sc->k; nothing for k = 1);
// q 1: p.Ap(k) before update k (k = sc->niters).
__global__ void __launch_bounds__(kBlock) fused_post_kernel(const double *parts, unsigned n,
                                                             const double *fallback, const PeerTab *t,
                                                             const CgScalars *sc, int q) {
    __shared__ double sh[33];
    pdl_wait();
    pdl_trigger();
    const int k = q == 0 ? ldg_o(&sc->k) - 1 : ldg_o(&sc->niters);
    if (q == 0 && k < 1) return;
    const double v = parts ? sum_parts_fixed(parts, n, sh) : __ldcg(fallback);
    if (threadIdx.x == 0)
        fused_post(t, q, v, ll_tag(ldg_o(&sc->epoch), q == 0 ? 2ull * (unsigned)k : 2ull * (unsigned)k - 1ull));
}

// deferred x update, end of the solve: the last iteration's x += alpha p (no p
// update followed it).  Nothing when no iteration ran.  Same FMA as the x/r
// update would have done, so the solution's bits do not depend on deferral.
__global__ void __launch_bounds__(kBlock) cg_xfix_kernel(int64_t n, double *x, const double *p,
                                                         const CgScalars *sc) {
    pdl_wait();
    if (ldg_o(&sc->niters) < 1) return;
    const double alpha = ldg_o(&sc->alpha_x);
    const int64_t tid = gtid(), nth = gnth(), nv = n >> 1;
    double2 *__restrict__ x2 = reinterpret_cast<double2 *>(x);
    const double2 *__restrict__ p2 = reinterpret_cast<const double2 *>(p);
    for (int64_t i = tid; i < nv; i += nth) {
        double2 xv = x2[i];
        const double2 pv = p2[i];
        xv.x = fma(alpha, pv.x, xv.x);
        xv.y = fma(alpha, pv.y, xv.y);
        x2[i] = xv;
    }
    if (tid == 0 && (n & 1)) x[n - 1] = fma(alpha, p[n - 1], x[n - 1]);
}

// ---- a.6 with the x update deferred over m iterations (HPCCG_OPT_DEFER_X =
// m >= 2, single slab).  x_k = x_(k-1) + alpha_k p_k is applied m iterations
// at a time: p_k of iteration k is written to ring slot k % (m + 1) (slot 0 is
// the problem's p buffer, the SpMV gathers from the slot of sc->k), so the m
// directions since the last flush stay in HBM, and the p update of iteration
// K with (K - 1) % m == 0 reads them once more and applies
//   x = fma(alpha_j, p_j, x),  j = K - m, ..., K - 1 (ascending)
// -- the FMAs the per-iteration update does, on the same operands in the same
// order, so x is bitwise identical.  Per m iterations the x stream costs one
// read and one write (16n B) plus m - 1 re-reads of old p (8n B each) instead
// of m reads and m writes: the reads stay 3 per iteration, the writes drop
// from 2 to 1 + 1/m (measured, tools/ringbench.cu: 2R:1W ring + one flush per
// m against 3R:2W in place).  cg_xfix_ring_kernel applies the pending ones
// after the loop.
constexpr int kRingMaxM = 8;

struct PRing {
    double *base;    // slot 1 (slot j >= 1 at base + (j - 1) stride; slot 0: the kernel's p)
    int64_t stride;  // doubles between slots
    int m;           // deferral depth: m + 1 slots
};

__device__ __forceinline__ double *ring_slot(double *p0, const PRing &g, int j) {
    return j == 0 ? p0 : g.base + (int64_t)(j - 1) * g.stride;
}

struct PringArgs {
    int64_t n;
    const double *r;
    double *p;  // slot 0 (owned part)
    PRing ring; // owned-part bases
    double *x;
    const double *rr_parts;
    unsigned n_rr;
    CgScalars *sc;
    int q;
    TraceSlot *trace;
    int trace_max;
    int rev;
    // HALO_PEER = 2 on z-slabs (kPeer): as Pupd1Args, the boundary planes of
    // p_K pushed into slot K % (m + 1) of the neighbours' rings; n_push / n_push1:
    // blocks holding a boundary row in the double2 / the flush (one element
    // per thread) mapping
    const PeerTab *t;
    int64_t plane;
    unsigned n_push, n_push1;
    int post;
};

// the neighbour halo plane of ring slot j (slot 0: the problem's p buffer)
__device__ __forceinline__ double *ring_peer_plane(double *slot0, double *slot1, int64_t stride, int j) {
    if (!slot0) return nullptr;
    return j == 0 ? slot0 : slot1 + (int64_t)(j - 1) * stride;
}

// the scalar part of p update K (after the PDL wait): beta, and block 0's
// loop state; false: iteration K does not run (uniform exit)
template <bool kPeer>
__device__ __forceinline__ bool ring_scalars(const PringArgs &a, int K, bool first, double *sh, double *beta) {
    CgScalars *sc = a.sc;
    if (!run_check(sc, a.q)) return false;
    trace_mark(a.trace, a.trace_max, K, 0, false);
    double rtrans = first ? ldg_o(&sc->rr_cur) : sum_parts_fixed(a.rr_parts, a.n_rr, sh);
    if (kPeer && !first) {  // z-slabs: the slab's r.r -> every rank; the global sum back
        const unsigned tag = ll_tag(ldg_o(&sc->epoch), 2ull * (unsigned)(K - 1));
        if (a.post && blockIdx.x == 0 && threadIdx.x == 0) fused_post(a.t, 0, rtrans, tag);
        rtrans = fused_collect_block(a.t, 0, tag, rtrans, &sh[32]);
    }
    *beta = first ? 0.0 : rtrans / ldg_o(&sc->rr_prev);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (!first) sc->rr_cur = rtrans;
        sc->normr = sqrt(rtrans);
        sc->niters = K;
        sc->ring_k[a.q] = K;
    }
    return true;
}

// flush iteration (K - 1 divisible by m): one double per thread per trip
// (scalar: the m + 2 loads in flight per thread fit the normal path's
// register budget); x, p_(K-1) and the m - 1 older directions are loaded
// before the wait
template <bool kPeer>
__device__ __forceinline__ void ring_flush(const PringArgs &a, int K, double *sh) {
    const int m = a.ring.m, R = m + 1;
    const int64_t tid = gtid(), nth = gnth(), n = a.n;
    const double *src = ring_slot(a.p, a.ring, (K - 1) % R);
    double *dst = ring_slot(a.p, a.ring, K % R);
    const double *__restrict__ r = a.r;
    double *x = a.x;
    // the older directions' slots (K - m + t) % R, t < m - 1
    __shared__ const double *sop[kRingMaxM - 1];
    if (threadIdx.x < kRingMaxM - 1)
        sop[threadIdx.x] =
            (int)threadIdx.x < m - 1 ? ring_slot(a.p, a.ring, (K - m + (int)threadIdx.x) % R) : nullptr;
    __syncthreads();
    const int64_t step = nth;
    const int64_t b0 = (a.rev && tid < n) ? tid + ((n - 1 - tid) / step) * step : tid;
    double pa = 0.0, ra = 0.0, xa = 0.0, oa[kRingMaxM - 1];
    auto ld_old = [&](int64_t i) {
        xa = x[i];
        pa = src[i];
#pragma unroll
        for (int t = 0; t < kRingMaxM - 1; ++t)
            if (t < m - 1) oa[t] = sop[t][i];
    };
    if (b0 < n) ld_old(b0);
    pdl_wait();
    pdl_trigger();
    if (b0 < n) ra = r[b0];
    double beta;
    if (!ring_scalars<kPeer>(a, K, false, sh, &beta)) return;
    double *plo = nullptr, *phi = nullptr;
    if (kPeer) {
        plo = ring_peer_plane(a.t->halo_to_lo, a.t->ring_to_lo, a.ring.stride, K % R);
        phi = ring_peer_plane(a.t->halo_to_hi, a.t->ring_to_hi, a.ring.stride, K % R);
    }
    int pushed = 0;
    __shared__ double sal[kRingMaxM];
    if (threadIdx.x < kRingMaxM)
        sal[threadIdx.x] = (int)threadIdx.x < m ? ldg_o(&a.sc->alpha_h[(K - m + (int)threadIdx.x) & 15]) : 0.0;
    __syncthreads();
    const double am = sal[m - 1];
    for (int64_t b = b0; b >= 0 && b < n;) {
        // x += alpha_j p_j, j = K - m .. K - 1 in ascending order (p_(K-1) = pa)
#pragma unroll
        for (int t = 0; t < kRingMaxM - 1; ++t)
            if (t < m - 1) xa = fma(sal[t], oa[t], xa);
        x[b] = fma(am, pa, xa);
        const double v = fma(beta, pa, ra);
        dst[b] = v;
        if (kPeer) {
            if (plo && b < a.plane) {
                plo[b] = v;
                pushed = 1;
            }
            if (phi && b >= n - a.plane) {
                phi[b - (n - a.plane)] = v;
                pushed = 1;
            }
        }
        b += a.rev ? -step : step;
        if (b >= 0 && b < n) {
            ra = r[b];
            ld_old(b);
        }
    }
    if (a.trace) {
        __syncthreads();
        trace_mark(a.trace, a.trace_max, K, 0, true);
    }
    if (kPeer) fused_push_signal(a.t, pushed, a.n_push1, ftag(ldg_o(&a.sc->epoch), (unsigned long long)K));
}

// (__launch_bounds__(kBlock, 3): the flush path's loads must not push the
// kernel past the 80 registers of cg_pupdate1_kernel<4>)

template <int kU, bool kPeer = false>
__global__ void __launch_bounds__(kBlock, 3) cg_pupdate_ring_kernel(PringArgs a) {
    __shared__ double sh[33];
    // this iteration's index from the p update before it (ring_k[q ^ 1],
    // written by p update K - 1, which completed before this grid's PDL
    // predecessor began): the slots are known before the wait
    // (ld.relaxed.gpu: a coherent read at GPU scope, never a stale L1 line -- it
    // precedes the wait, so the PDL visibility guarantee does not cover it)
    int kprev;
    asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(kprev) : "l"(&a.sc->ring_k[a.q ^ 1]) : "memory");
    const int K = kprev + 1;
    const int m = a.ring.m, R = m + 1;
    const bool first = (K == 1);
    if (!first && (K - 1) % m == 0) {
        ring_flush<kPeer>(a, K, sh);
        return;
    }
    const int64_t tid = gtid(), nth = gnth(), nv = a.n >> 1;
    // plain loads (no const __restrict__): the first ones precede the PDL wait
    const double *srcd = ring_slot(a.p, a.ring, (K - 1) % R);
    double *dstd = ring_slot(a.p, a.ring, K % R);
    const double2 *src = reinterpret_cast<const double2 *>(srcd);
    double2 *dst = reinterpret_cast<double2 *>(dstd);
    const double2 *__restrict__ r2 = reinterpret_cast<const double2 *>(a.r);
    const int64_t step = kU * nth;
    const int64_t b0 = (a.rev && tid < nv) ? tid + ((nv - 1 - tid) / step) * step : tid;
    double2 ra[kU], pa[kU];
    auto load_p = [&](int64_t b) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < nv) pa[u] = ld_hint<8>(src + i);
        }
    };
    auto load_r = [&](int64_t b) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < nv) ra[u] = ld_hint<8>(r2 + i);
        }
    };
    if (!first) load_p(b0);
    pdl_wait();
    pdl_trigger();
    load_r(b0);
    double beta;
    if (!ring_scalars<kPeer>(a, K, first, sh, &beta)) return;
    const int64_t n = a.n;
    double *plo = nullptr, *phi = nullptr;
    if (kPeer) {
        plo = ring_peer_plane(a.t->halo_to_lo, a.t->ring_to_lo, a.ring.stride, K % R);
        phi = ring_peer_plane(a.t->halo_to_hi, a.t->ring_to_hi, a.ring.stride, K % R);
    }
    int pushed = 0;
    auto put = [&](int64_t i, double v) {  // row i of p_K -> a neighbour's halo (slot K % R)
        if (plo && i < a.plane) {
            plo[i] = v;
            pushed = 1;
        }
        if (phi && i >= n - a.plane) {
            phi[i - (n - a.plane)] = v;
            pushed = 1;
        }
    };
    for (int64_t b = b0; b >= 0 && b < nv;) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < nv) {
                double2 v = ra[u];
                if (!first) {
                    v.x = fma(beta, pa[u].x, ra[u].x);
                    v.y = fma(beta, pa[u].y, ra[u].y);
                }
                st_p(dst + i, v);
                if (kPeer && (2 * i < a.plane || 2 * i + 1 >= n - a.plane)) {
                    put(2 * i, v.x);
                    put(2 * i + 1, v.y);
                }
            }
        }
        b += a.rev ? -step : step;
        if (b >= 0 && b < nv) {
            load_r(b);
            if (!first) load_p(b);
        }
    }
    if (tid == 0 && (a.n & 1)) {
        const int64_t i = a.n - 1;
        const double v = first ? a.r[i] : fma(beta, srcd[i], a.r[i]);
        dstd[i] = v;
        if (kPeer) put(i, v);
    }
    if (a.trace) {
        __syncthreads();
        trace_mark(a.trace, a.trace_max, K, 0, true);
    }
    if (kPeer) fused_push_signal(a.t, pushed, a.n_push, ftag(ldg_o(&a.sc->epoch), (unsigned long long)K));
}

// end of a solve with the ring-deferred x update: the directions since the
// last flush, j = F + 1 .. N with F = m floor((N - 1) / m) and N = niters (p
// update N flushed up to N - 1 only when m divides N - 1), in ascending order
// shift: 1 for HPCCG's loop (p update K flushes up to K - 1), 0 for f2's
// (update k flushes up to k itself)
__global__ void __launch_bounds__(kBlock) cg_xfix_ring_kernel(int64_t n, double *x, double *p0, PRing g,
                                                              const CgScalars *sc, int shift) {
    pdl_wait();
    const int N = ldg_o(&sc->niters);
    if (N < 1) return;
    const int m = g.m, R = m + 1, F = m * ((N - shift) / m), c = N - F;
    if (c <= 0) return;
    const double *pj[kRingMaxM];
    double al[kRingMaxM];
#pragma unroll
    for (int t = 0; t < kRingMaxM; ++t) {
        pj[t] = t < c ? ring_slot(p0, g, (F + 1 + t) % R) : nullptr;
        al[t] = t < c ? ldg_o(&sc->alpha_h[(F + 1 + t) & 15]) : 0.0;
    }
    const int64_t tid = gtid(), nth = gnth(), nv = n >> 1;
    double2 *__restrict__ x2 = reinterpret_cast<double2 *>(x);
    for (int64_t i = tid; i < nv; i += nth) {
        double2 xv = x2[i];
#pragma unroll
        for (int t = 0; t < kRingMaxM; ++t) {
            if (t < c) {
                const double2 pv = reinterpret_cast<const double2 *>(pj[t])[i];
                xv.x = fma(al[t], pv.x, xv.x);
                xv.y = fma(al[t], pv.y, xv.y);
            }
        }
        x2[i] = xv;
    }
    if (tid == 0 && (n & 1)) {
        double xv = x[n - 1];
#pragma unroll
        for (int t = 0; t < kRingMaxM; ++t)
            if (t < c) xv = fma(al[t], pj[t][n - 1], xv);
        x[n - 1] = xv;
    }
}

// ---- a.6 + a.3 + a.4 fused and pipelined (HPCCG_OPT_FUSE_PSPMV): the p
// update of iteration k and the SpMV Ap = A p_k in ONE kernel, single slab.
// Chunk c = rows [512c, 512c + 512) (one 256-thread block's SpMV rows, 2 per
// thread, the partial slot c of the unfused SpMV: identical bits).  Blocks take
// tickets t in launch order (an atomic counter) and SpMV the chunk at position
// t (pos reverses the chunk order under serpentine).  Block t first applies p =
// r + beta p (and the deferred x += alpha_x p) to the chunk at position t +
// lead and publishes it with a release flag; the chunks at positions < lead
// were updated by the p-update kernel launched just before (cg_pupdate1_kernel
// on those rows only).  Its SpMV then waits (acquire) for the <= 9 chunks its
// gathers touch (the z-1, z, z+1 windows), all at positions < t + lead when
// lead > plane/512 + 2, i.e. produced by the prologue or by EARLIER tickets
// that publish before they wait: no block ever waits for a block that has not
// started, so the kernel cannot deadlock whatever the residency.  p_k is
// gathered from L2 a few microseconds after it is written: the SpMV's 8n B read
// of p from HBM goes (12 nnz + 72n B per iteration with the deferred x update,
// instead of 80n).  The gathers are weak L1-cached loads: a line of p belongs
// to one chunk (the host checks the alignment) and is first read after the
// flag acquire (which invalidates the SM's L1), so no SM holds a stale copy;
// p_old is read with L1::no_allocate.
constexpr int kPsRows = 2 * kBlock;  // rows per chunk

struct PsArgs {
    int64_t n, plane, nchunks;
    int nx, lead, rev, q;
    const double *val;
    const int *col;
    double *p;                    // local-with-halo base: p[plane + i] is row i
    const double *r;
    double *x;                    // deferred x update (nullptr: none)
    double *Ap;
    double *parts;                // out: per-chunk p.Ap partials (chunk order)
    const double *rr_parts;       // r.r partials of the previous update
    unsigned n_rr;
    CgScalars *sc;
    unsigned *ticket;             // launch-order counter (reset by the last ticket)
    unsigned long long *flags;    // [nchunks] chunk c of p_k published: tag(epoch, k)
    TraceSlot *trace;
    int trace_max;
    int *err;                     // a wait that gave up (5 s): the solve reports HPCCG_ECUDA
};

__device__ __forceinline__ void st_release_gpu(unsigned long long *p, unsigned long long v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_gpu(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_relaxed_gpu(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ double2 ld_na2(const double2 *p) {  // coherent, no L1 allocation
    double2 v;
    asm volatile("ld.global.L1::no_allocate.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p) : "memory");
    return v;
}

// wait until *f >= tag with acquire semantics: one acquire load in the common
// case; else relaxed polls and a final acquire; gives up after 5 s (only a bug
// could get there) with *err set instead of hanging the GPU
__device__ __forceinline__ void ps_wait(const PsArgs &a, const unsigned long long *f, unsigned long long tag) {
    if (ld_acquire_gpu(f) >= tag) return;
    const unsigned long long t0 = gtimer();
    while (ld_relaxed_gpu(f) < tag) {
        if (*(volatile int *)a.err || gtimer() - t0 > 5000000000ull) {
            *(volatile int *)a.err = 1;
            return;
        }
        __nanosleep(64);
    }
    (void)ld_acquire_gpu(f);
}

__global__ void __launch_bounds__(kBlock, 4) cg_pspmv_kernel(PsArgs a) {
    __shared__ unsigned s_t;
    __shared__ double shp[33];
    if (threadIdx.x == 0) s_t = atomicAdd(a.ticket, 1u);
    __syncthreads();
    const unsigned t = s_t;
    if (threadIdx.x == 0 && t == (unsigned)a.nchunks - 1u) *a.ticket = 0u;  // every ticket taken
    const int64_t c = a.rev ? a.nchunks - 1 - (int64_t)t : (int64_t)t;
    const int64_t row = c * kPsRows + 2 * threadIdx.x;
    const bool active = row < a.n;  // n even: both rows of the pair exist
    const uint64_t pol = policy_evict_first();
    const double *v = a.val + row;
    const int *ci = a.col + row;
    // the matrix does not depend on the predecessor: the first group's loads
    // are in flight before the PDL wait and the producer work
    double2 vv0[3];
    int2 cc0[3];
    if (active) {
#pragma unroll
        for (int u = 0; u < 3; ++u) {
            vv0[u] = ld_stream2(v + u * a.n, pol);
            cc0[u] = ld_stream2(ci + u * a.n, pol);
        }
    }
    pdl_wait();
    if (!ldp(&a.sc->run_q[a.q ^ 1])) {  // uniform: iteration k does not run (run_check)
        if (t == 0 && threadIdx.x == 0) a.sc->run_q[a.q] = 0;
        return;
    }
    CgScalars *sc = a.sc;
    const int k = ldp(&sc->k);
    const bool first = (k == 1);
    const unsigned long long tag = ftag(ldp(&sc->epoch), (unsigned long long)k);
    trace_mark(a.trace, a.trace_max, k, 1, false);
    pdl_trigger();
    // produce the chunk `lead` positions ahead (beta / alpha_x were finished
    // and stored by the prologue p update's block 0: ordered loads after the wait)
    const int64_t tp = (int64_t)t + a.lead;
    if (tp < a.nchunks) {
        const double beta = first ? 0.0 : ldp(&sc->rr_cur) / ldp(&sc->rr_prev);
        const double alpha_x = first ? 0.0 : ldp(&sc->alpha_x);
        const int64_t cp = a.rev ? a.nchunks - 1 - tp : tp;
        const int64_t i = (cp * kPsRows >> 1) + threadIdx.x;  // 16-B unit
        if (2 * i < a.n) {
            double2 *p2 = reinterpret_cast<double2 *>(a.p + a.plane);
            const double2 rv = ldp(reinterpret_cast<const double2 *>(a.r) + i);
            double2 pv = rv;
            if (!first) {
                const double2 po = ld_na2(p2 + i);
                pv.x = fma(beta, po.x, rv.x);
                pv.y = fma(beta, po.y, rv.y);
                if (a.x) {
                    double2 *x2 = reinterpret_cast<double2 *>(a.x);
                    double2 xv = ld_na2(x2 + i);
                    xv.x = fma(alpha_x, po.x, xv.x);
                    xv.y = fma(alpha_x, po.y, xv.y);
                    x2[i] = xv;
                }
            }
            p2[i] = pv;
        }
        __syncthreads();  // the block's stores before thread 0's release (cumulative)
        if (threadIdx.x == 0) st_release_gpu(a.flags + cp, tag);
    }
    // consume: wait for the chunks this block's gathers read (z-1, z, z+1
    // windows of rows [512c - nx - 1, 512c + 511 + nx + 1]); thread 3w + o
    // takes chunk o of window w, all polls in flight at once
    if (threadIdx.x < 9) {
        const int w = threadIdx.x / 3, o = threadIdx.x % 3;
        const int64_t lo = c * kPsRows + (w - 1) * a.plane - a.nx - 1;
        const int64_t hi = c * kPsRows + kPsRows - 1 + (w - 1) * a.plane + a.nx + 1;
        const int64_t l = max(lo, (int64_t)0), h = min(hi, a.n - 1);
        const int64_t cw = l / kPsRows + o;
        if (l <= h && cw <= h / kPsRows) {
            const int64_t pw = a.rev ? a.nchunks - 1 - cw : cw;  // its position
            if (pw >= a.lead) ps_wait(a, a.flags + cw, tag);  // else: the prologue's
        }
    }
    __syncthreads();
    double d = 0.0;
    if (active) {
        const double *px = a.p;
        double s0 = 0.0, s1 = 0.0, x0 = 0.0, x1 = 0.0;
        int c0 = 0, c1 = 0;
#pragma unroll
        for (int g = 0; g < kSlots / 3; ++g) {
            double2 vv[3];
            int2 cc[3];
#pragma unroll
            for (int u = 0; u < 3; ++u) {
                if (g == 0) {
                    vv[u] = vv0[u];
                    cc[u] = cc0[u];
                } else {
                    vv[u] = ld_stream2(v + (3 * g + u) * a.n, pol);
                    cc[u] = ld_stream2(ci + (3 * g + u) * a.n, pol);
                }
            }
#pragma unroll
            for (int u = 0; u < 3; ++u) {
                const double xa = px[cc[u].x], xb = px[cc[u].y];  // weak, L1-cached (see above)
                if (3 * g + u == kDiagSlot) {
                    x0 = xa;
                    x1 = xb;
                    c0 = cc[u].x;
                    c1 = cc[u].y;
                }
                s0 = fma(vv[u].x, xa, s0);
                s1 = fma(vv[u].y, xb, s1);
            }
        }
        *reinterpret_cast<double2 *>(a.Ap + row) = make_double2(s0, s1);
        const double p0 = c0 == row + a.plane ? x0 : px[row + a.plane];
        const double p1 = c1 == row + 1 + a.plane ? x1 : px[row + 1 + a.plane];
        d = fma(s1, p1, s0 * p0);
    }
    d = block_reduce<false>(d, shp);
    if (threadIdx.x == 0) a.parts[c] = d;
    trace_mark(a.trace, a.trace_max, k, 1, true);
}

template <int kU, bool kPeer = false, bool kLateP = false>
__global__ void __launch_bounds__(kBlock) cg_update1_kernel(Upd1Args a) {
    __shared__ double sh[33];
    CgScalars *sc = a.sc;
    const int64_t tid = gtid(), nth = gnth(), nv = a.n >> 1;
    double2 *__restrict__ x2 = reinterpret_cast<double2 *>(a.x);
    double2 *__restrict__ r2 = reinterpret_cast<double2 *>(a.r);
    const double2 *__restrict__ p2 = reinterpret_cast<const double2 *>(a.p);
    const double2 *__restrict__ q2 = reinterpret_cast<const double2 *>(a.Ap);
    double2 xa[kU], ra[kU], pa[kU], qa[kU];
    const bool dx = a.defer_x != 0;
    auto load_xrp = [&](int64_t b) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < nv) {
                ra[u] = r2[i];
                if (!dx) {
                    xa[u] = x2[i];
                    pa[u] = p2[i];
                }
            }
        }
    };
    auto load_q = [&](int64_t b) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < nv) qa[u] = ld_hint<16>(q2 + i);
        }
    };
    auto load = [&](int64_t b) {
        load_xrp(b);
        load_q(b);
    };
    // x, r (previous update) and p (p update) are complete before the SpMV's
    // blocks pass their pdl_wait, so before this grid can launch: read them
    // during the SpMV's tail; Ap only after the SpMV has completed.  Fused p
    // update + SpMV: p (and x) come from the predecessor itself -> after the wait
    const bool early = !(kLateP && !dx);
    if (early) load_xrp(tid);
    pdl_wait();
    pdl_trigger();
    if (!early) load_xrp(tid);
    load_q(tid);
    if (!run_check(sc, a.q)) return;
    const int ktr = a.trace ? ldg_o(&sc->niters) : 0;
    trace_mark(a.trace, a.trace_max, ktr, 2, false);
    const double rtrans = ldg_o(&sc->rr_cur);
    double pAp = a.pAp_parts ? sum_parts_fixed(a.pAp_parts, a.n_parts, sh) : ldg_o(&sc->pAp);
    if (kPeer) {  // z-slabs: the slab's p.Ap -> every rank; the global sum back
        const unsigned tag = ll_tag(ldg_o(&sc->epoch), 2ull * (unsigned)ldg_o(&sc->niters) - 1ull);
        if (a.post && blockIdx.x == 0 && threadIdx.x == 0) fused_post(a.t, 1, pAp, tag);
        pAp = fused_collect_block(a.t, 1, tag, pAp, &sh[32]);
    }
    const bool stop = (rtrans == 0.0) || (pAp == 0.0);  // A11
    const double alpha = stop ? 0.0 : rtrans / pAp;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        const int k = ldg_o(&sc->k);
        const int run = !stop && (k + 1) < ldg_o(&sc->max_iter) && ldg_o(&sc->normr) > ldg_o(&sc->tol);
        sc->pAp = pAp;
        sc->rr_prev = rtrans;
        sc->alpha_x = alpha;
        sc->alpha_h[k & 15] = alpha;
        sc->k = k + 1;
        sc->run_q[a.q] = run;
        sc->done = !run;
        set_cond(a.cond, run);
    }
    double acc = 0.0, acc2 = 0.0;
    for (int64_t b = tid; b < nv;) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < nv) {
                if (!dx) {
                    xa[u].x = fma(alpha, pa[u].x, xa[u].x);
                    xa[u].y = fma(alpha, pa[u].y, xa[u].y);
                    x2[i] = xa[u];
                }
                ra[u].x = fma(-alpha, qa[u].x, ra[u].x);
                ra[u].y = fma(-alpha, qa[u].y, ra[u].y);
                st_hint<4>(r2 + i, ra[u]);
                acc = fma(ra[u].x, ra[u].x, acc);
                acc2 = fma(ra[u].y, ra[u].y, acc2);
            }
        }
        b += kU * nth;
        if (b < nv) load(b);
    }
    if (tid == 0 && (a.n & 1)) {
        const int64_t i = a.n - 1;
        if (!dx) a.x[i] = fma(alpha, a.p[i], a.x[i]);
        const double rv = fma(-alpha, a.Ap[i], a.r[i]);
        a.r[i] = rv;
        acc = fma(rv, rv, acc);
    }
    acc += acc2;
    trace_mark(a.trace, a.trace_max, ktr, 2, true);
    acc = block_reduce<false>(acc, sh);
    if (threadIdx.x == 0) a.rr_parts[blockIdx.x] = acc;
}

// a.7 init: r = b - Ap (waxpby(1, b, -1, Ap) = fma(-1, Ap, b)) and r.r.
struct InitResArgs {
    int64_t n;
    const double *b, *Ap;
    double *r;
    CgScalars *sc;
    Reduction red;
    int single;
};

__global__ void __launch_bounds__(kBlock) cg_initres_kernel(InitResArgs a) {
    const int64_t tid = gtid(), nth = gnth();
    double acc = 0.0;
    for (int64_t i = tid; i < a.n; i += nth) {
        const double rv = fma(-1.0, a.Ap[i], a.b[i]);
        a.r[i] = rv;
        acc = fma(rv, rv, acc);
    }
    CgScalars *sc = a.sc;
    const int single = a.single;
    grid_reduce<false>(acc, a.red, blockIdx.x, gridDim.x, [sc, single](double s) {
        if (single) sc->rr_cur = s; else sc->loc_rr = s;
    });
}

// a.7/a.8: after the (allreduced) initial r.r: k = 1, normr, first check.
__global__ void cg_initstate_kernel(CgScalars *sc, int max_iter, double tol,
                                    unsigned long long cond) {
    const double rr = sc->rr_cur;
    const double normr = sqrt(rr);
    sc->rr_prev = rr;
    sc->normr = normr;
    sc->tol = tol;
    sc->max_iter = max_iter;
    sc->k = 1;
    sc->niters = 0;
    const int done = !(1 < max_iter && normr > tol);
    sc->done = done;
    sc->run_q[0] = !done;  // finisher-free loop: iteration 1 (parity 1) runs
    sc->run_q[1] = 0;
    sc->ring_k[0] = 0;  // ring-deferred x update: p update 1 (parity 1) reads ring_k[0]
    sc->ring_k[1] = 0;
    sc->epoch = sc->epoch + 1;
    set_cond(cond, !done);
}

// ------------------------------- f2: single-reduction (Chronopoulos-Gear) CG
// Same HPCCG loop control (A4 lag, A11 guard) as the kernels above; the
// iteration is two kernels: this fused update, then the SpMV w = A r with the
// (gamma, delta) epilogue (spmv27*_kernel<2>).  The update of iteration k
//   beta = gamma / gamma_old, den = delta - (beta gamma) / alpha_old
//   (k = 1: beta = 0, den = delta), alpha = gamma / den
//   p = r + beta p; s = w + beta s; x = x + alpha p; r = r - alpha s
// makes ONE pass over r, w, p, s, x (reads 5, writes 4: 72n B, the same bytes
// as HPCCG's p update + x/r update) and needs no grid-wide reduction of its
// own: every block sums the previous SpMV's (gamma, delta) partials in the
// same fixed order, so every block holds bit-identical scalars, and block 0
// writes the double-buffered loop state (CgScalars::sr_*).  The scalar
// arithmetic uses explicit round-to-nearest intrinsics in the oracle's
// order (no contraction), so it matches oracle_cg_sr step for step.
// Multi-slab: a finisher sums the partials into loc_gd, one allreduce of
// the two values gives gd (one collective per iteration instead of two).

struct SrUpdArgs {
    int64_t n;
    double *x, *r, *p, *s;     // r: owned part of the gathered (halo) vector
    // x deferred over ring.m >= 2 iterations (HPCCG_OPT_DEFER_X): p_k in slot
    // k % (m + 1) (slot 0 = p), x += alpha_j p_j for the last m directions in
    // the update with k % m == 0 (the same FMAs in the same order); m < 2: none
    PRing ring;
    const double *w;
    const double *parts;       // non-null: (gamma, delta) = fixed-order sums of
    unsigned n_parts;          //   parts[0, n_parts) and parts[n_parts, 2 n_parts)
    CgScalars *sc;
    int q;                     // parity of the iteration this launch runs
    unsigned long long cond;   // while-graph condition handle (0: none)
    // HALO_PEER = 2 on z-slabs (kPeer): (gamma, delta) = the P slabs' sums
    // (k > 1; block 0 posts this slab's unless `post` is 0), and the first /
    // last owned plane of the new r pushed into the neighbours' halos
    const PeerTab *t;
    int64_t plane;
    unsigned n_push;
    unsigned n_push1;  // pushing blocks of the ring flush pass (one element per thread per trip)
    int post;
};

// Fixed-order sums of the (gamma, delta) partials, identical in every block.
__device__ __forceinline__ double2 sr_sum_parts(const double *parts, unsigned np, double *sh) {
    double g = 0.0, d = 0.0;
    unsigned i = threadIdx.x;
    for (; i + 3u * kBlock < np; i += 4u * kBlock) {  // 8 loads in flight
        double vg[4], vd[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            vg[u] = ldg_o(parts + i + u * kBlock);
            vd[u] = ldg_o(parts + np + i + u * kBlock);
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            g += vg[u];
            d += vd[u];
        }
    }
    for (; i < np; i += kBlock) {
        g += ldg_o(parts + i);
        d += ldg_o(parts + np + i);
    }
    double2 t = block_reduce2(g, d, sh);
    if (threadIdx.x == 0) {
        sh[64] = t.x;
        sh[65] = t.y;
    }
    __syncthreads();
    t = make_double2(sh[64], sh[65]);
    return t;
}

// (gamma, delta) partials of one slab -> out[0..1] (one block, fixed order):
// multi-slab (allreduce input) or a single slab with > kUpdSumMax partials.
// 1024 threads, 8 loads in flight per thread (65536 partials at 256^3).
__global__ void __launch_bounds__(1024, 1) cg_sr_finish_kernel(const double *parts, unsigned n_parts,
                                                            double *out) {
    pdl_wait();
    pdl_trigger();
    __shared__ double sh[64];
    double g[4] = {0.0, 0.0, 0.0, 0.0}, d[4] = {0.0, 0.0, 0.0, 0.0};
    unsigned i = threadIdx.x;
    // 3 trips' loads in flight, added trip by trip (same order as below)
    for (; i + 11u * 1024u < n_parts; i += 12u * 1024u) {
        double vg[12], vd[12];
#pragma unroll
        for (int u = 0; u < 12; ++u) {
            vg[u] = ldg_o(parts + i + u * 1024u);
            vd[u] = ldg_o(parts + n_parts + i + u * 1024u);
        }
#pragma unroll
        for (int t = 0; t < 3; ++t)
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                g[u] += vg[4 * t + u];
                d[u] += vd[4 * t + u];
            }
    }
    for (; i + 3u * 1024u < n_parts; i += 4u * 1024u) {
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            g[u] += __ldcg(parts + i + u * 1024u);
            d[u] += __ldcg(parts + n_parts + i + u * 1024u);
        }
    }
    for (; i < n_parts; i += 1024u) {
        g[0] += __ldcg(parts + i);
        d[0] += __ldcg(parts + n_parts + i);
    }
    double gs = (g[0] + g[1]) + (g[2] + g[3]), ds = (d[0] + d[1]) + (d[2] + d[3]);
    gs = warp_sum(gs);
    ds = warp_sum(ds);
    if ((threadIdx.x & 31) == 0) {
        sh[threadIdx.x >> 5] = gs;
        sh[32 + (threadIdx.x >> 5)] = ds;
    }
    __syncthreads();
    if (threadIdx.x < 32) {
        gs = warp_sum(sh[threadIdx.x]);
        ds = warp_sum(sh[32 + threadIdx.x]);
        if (threadIdx.x == 0) {
            out[0] = gs;
            out[1] = ds;
        }
    }
}

// Loopback + HALO_PEER = 2, f2: post a slab's (gamma, delta) of the previous
// SpMV ahead of every update (see fused_post_kernel).  q: the parity of the
// update about to run; nothing for its first iteration.
__global__ void __launch_bounds__(kBlock) fused_post2_kernel(const double *parts, unsigned n,
                                                              const double *fallback, const PeerTab *t,
                                                              const CgScalars *sc, int q) {
    __shared__ double sh[66];
    pdl_wait();
    pdl_trigger();
    const int k = ldg_o(&sc->sr_k[q ^ 1]);
    if (k < 2 || !ldg_o(&sc->run_q[q ^ 1])) return;
    const double2 v = parts ? sr_sum_parts(parts, n, sh) : make_double2(__ldcg(fallback), __ldcg(fallback + 1));
    if (threadIdx.x == 0) fused_post2(t, (k - 1) & 1, v, ll_tag(ldg_o(&sc->epoch), (unsigned)(k - 1)));
}

template <bool kVec, int kU, bool kPeer = false>
__global__ void __launch_bounds__(kBlock) cg_sr_update_kernel(SrUpdArgs a) {
    CgScalars *sc = a.sc;
    const int q = a.q, qp = q ^ 1;
    // r, p, s, x were written by the previous update, complete before the
    // SpMV's blocks passed their wait: warm L2/L1 with the first trip while
    // the SpMV drains (w, the SpMV's output, only after the wait)
    if (kVec) {
        const int64_t nv0 = a.n >> 1;
        for (int u = 0; u < kU; ++u) {
            const int64_t i = gtid() + u * gnth();
            if (i < nv0) {
                asm volatile("prefetch.global.L2 [%0];" ::"l"(a.r + 2 * i));
                if (a.ring.m < 2) {  // (with the ring: p's slot is known only after the wait, x unused)
                    asm volatile("prefetch.global.L2 [%0];" ::"l"(a.x + 2 * i));
                    asm volatile("prefetch.global.L2 [%0];" ::"l"(a.p + 2 * i));
                }
                asm volatile("prefetch.global.L2 [%0];" ::"l"(a.s + 2 * i));
            }
        }
    }
    pdl_wait();
    pdl_trigger();
    if (!ldg_o(&sc->run_q[qp])) {  // iteration k does not run (uniform) ...
        // ... and neither does k + 1: propagate, or slot q would keep the stale
        // flag of iteration k - 1 for the launches of parity q that follow
        if (blockIdx.x == 0 && threadIdx.x == 0) sc->run_q[q] = 0;
        return;
    }
    __shared__ double sh[66];
    double2 gd;
    const int k = ldg_o(&sc->sr_k[qp]);
    const bool first = (k == 1);
    if (kPeer) {  // z-slabs: k = 1 takes the init's allreduced values
        if (first) {
            gd = make_double2(ldg_o(&sc->gd[0]), ldg_o(&sc->gd[1]));
        } else {
            gd = a.parts ? sr_sum_parts(a.parts, a.n_parts, sh)
                         : make_double2(__ldcg(&sc->loc_gd[0]), __ldcg(&sc->loc_gd[1]));
            const unsigned tag = ll_tag(ldg_o(&sc->epoch), (unsigned)(k - 1));
            if (a.post && blockIdx.x == 0 && threadIdx.x == 0) fused_post2(a.t, (k - 1) & 1, gd, tag);
            gd = fused_collect2_block(a.t, (k - 1) & 1, tag, gd, &sh[64]);
        }
    } else if (a.parts) {
        gd = sr_sum_parts(a.parts, a.n_parts, sh);
    } else {
        gd = make_double2(ldg_o(&sc->gd[0]), ldg_o(&sc->gd[1]));
    }
    const double gamma = gd.x, delta = gd.y;
    const double beta = first ? 0.0 : __ddiv_rn(gamma, ldg_o(&sc->sr_gamma[qp]));
    const double den =
        first ? delta : __dsub_rn(delta, __ddiv_rn(__dmul_rn(beta, gamma), ldg_o(&sc->sr_alpha[qp])));
    const bool stop = (gamma == 0.0) || (den == 0.0);  // A11
    const double alpha = stop ? 0.0 : __ddiv_rn(gamma, den);
    // the ring-deferred x update: this iteration's p source / destination slots
    const int rm = a.ring.m, rR = rm + 1;
    const bool ring = kVec && rm >= 2;
    double *psrc = ring ? ring_slot(a.p, a.ring, (k - 1) % rR) : a.p;
    double *pdst = ring ? ring_slot(a.p, a.ring, k % rR) : a.p;
    const bool flush = ring && (k % rm == 0);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        sc->alpha_h[k & 15] = alpha;
        const double normr = sqrt(gamma);  // ||r_(k-1)||: the lagged check (A4)
        const int nrun = !stop && (k + 1 < ldg_o(&sc->max_iter)) && normr > ldg_o(&sc->tol);
        sc->sr_gamma[q] = gamma;
        sc->sr_alpha[q] = alpha;
        sc->sr_k[q] = k + 1;
        sc->run_q[q] = nrun;
        sc->normr = normr;
        sc->niters = k;
        sc->done = !nrun;
        set_cond(a.cond, nrun);
    }
    const int64_t tid = gtid(), nth = gnth();
    double *lo = kPeer ? a.t->halo_to_lo : nullptr, *hi = kPeer ? a.t->halo_to_hi : nullptr;
    int pushed = 0;
    auto put = [&](int64_t i, double v) {  // row i of the new r -> a neighbour's halo
        if (lo && i < a.plane) {
            lo[i] = v;
            pushed = 1;
        }
        if (hi && i >= a.n - a.plane) {
            hi[i - (a.n - a.plane)] = v;
            pushed = 1;
        }
    };
    if (flush) {
        // x += alpha_j p_j, j = k - m + 1 .. k (p_k computed here): one element
        // per thread per trip, the m - 1 older directions from their slots
        __shared__ const double *sop[kRingMaxM - 1];
        __shared__ double sal[kRingMaxM];
        if (threadIdx.x < kRingMaxM) {
            const int t = threadIdx.x, j = k - rm + 1 + t;
            if (t < kRingMaxM - 1) sop[t] = t < rm - 1 ? ring_slot(a.p, a.ring, j % rR) : nullptr;
            sal[t] = t < rm ? ldg_o(&sc->alpha_h[j & 15]) : 0.0;
        }
        __syncthreads();
        const double ak = alpha;
        for (int64_t i = tid; i < a.n; i += nth) {
            double ov[kRingMaxM - 1];
            const double rv = a.r[i], wv = a.w[i], pv0 = psrc[i], sv0 = a.s[i];
            double xv = a.x[i];
#pragma unroll
            for (int t = 0; t < kRingMaxM - 1; ++t)
                if (t < rm - 1) ov[t] = sop[t][i];
            const double pv = first ? rv : fma(beta, pv0, rv);
            const double sv = first ? wv : fma(beta, sv0, wv);
#pragma unroll
            for (int t = 0; t < kRingMaxM - 1; ++t)
                if (t < rm - 1) xv = fma(sal[t], ov[t], xv);
            pdst[i] = pv;
            a.s[i] = sv;
            a.x[i] = fma(ak, pv, xv);
            const double rn = fma(-alpha, sv, rv);
            a.r[i] = rn;
            if (kPeer) put(i, rn);
        }
        if (kPeer) fused_push_signal(a.t, pushed, a.n_push1, ftag(ldg_o(&sc->epoch), (unsigned long long)k));
    } else if (kVec) {
        const int64_t nv = a.n >> 1;
        double2 *__restrict__ x2 = reinterpret_cast<double2 *>(a.x);
        double2 *__restrict__ r2 = reinterpret_cast<double2 *>(a.r);
        const double2 *ps2 = reinterpret_cast<const double2 *>(psrc);  // (slot (k - 1) % R with the ring)
        double2 *pd2 = reinterpret_cast<double2 *>(pdst);
        double2 *__restrict__ s2 = reinterpret_cast<double2 *>(a.s);
        const double2 *__restrict__ w2 = reinterpret_cast<const double2 *>(a.w);
        for (int64_t b = tid; b < nv; b += kU * nth) {
            double2 ra[kU], wa[kU], pa[kU], sa[kU], xa[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int64_t i = b + u * nth;
                if (i < nv) {
                    ra[u] = r2[i];
                    wa[u] = w2[i];
                    if (!first) {
                        pa[u] = ps2[i];
                        sa[u] = s2[i];
                    }
                    if (!ring) xa[u] = x2[i];
                }
            }
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int64_t i = b + u * nth;
                if (i < nv) {
                    double2 pv = ra[u], sv = wa[u];
                    if (!first) {
                        pv.x = fma(beta, pa[u].x, ra[u].x);
                        pv.y = fma(beta, pa[u].y, ra[u].y);
                        sv.x = fma(beta, sa[u].x, wa[u].x);
                        sv.y = fma(beta, sa[u].y, wa[u].y);
                    }
                    pd2[i] = pv;
                    s2[i] = sv;
                    if (!ring) x2[i] = make_double2(fma(alpha, pv.x, xa[u].x), fma(alpha, pv.y, xa[u].y));
                    const double2 rn = make_double2(fma(-alpha, sv.x, ra[u].x), fma(-alpha, sv.y, ra[u].y));
                    r2[i] = rn;
                    if (kPeer && (2 * i < a.plane || 2 * i + 1 >= a.n - a.plane)) {
                        put(2 * i, rn.x);
                        put(2 * i + 1, rn.y);
                    }
                }
            }
        }
        if (tid == 0 && (a.n & 1)) {
            const int64_t i = a.n - 1;
            const double pv = first ? a.r[i] : fma(beta, psrc[i], a.r[i]);
            const double sv = first ? a.w[i] : fma(beta, a.s[i], a.w[i]);
            pdst[i] = pv;
            a.s[i] = sv;
            if (!ring) a.x[i] = fma(alpha, pv, a.x[i]);
            a.r[i] = fma(-alpha, sv, a.r[i]);
            if (kPeer) put(i, a.r[i]);
        }
        if (kPeer) fused_push_signal(a.t, pushed, a.n_push, ftag(ldg_o(&sc->epoch), (unsigned long long)k));
    } else {
        for (int64_t i = tid; i < a.n; i += nth) {
            const double pv = first ? a.r[i] : fma(beta, a.p[i], a.r[i]);
            const double sv = first ? a.w[i] : fma(beta, a.s[i], a.w[i]);
            a.p[i] = pv;
            a.s[i] = sv;
            a.x[i] = fma(alpha, pv, a.x[i]);
            a.r[i] = fma(-alpha, sv, a.r[i]);
        }
    }
}

// f2 init, after w = A r0 and its (gamma, delta) partials (or gd): the loop
// state slot 0 (read by iteration k = 1, parity 1), normr = ||r0||, first
// check (A4).  One block.
__global__ void __launch_bounds__(kBlock) cg_sr_initstate_kernel(const double *parts, unsigned n_parts,
                                                                 CgScalars *sc, int max_iter,
                                                                 double tol, unsigned long long cond) {
    __shared__ double sh[66];
    double gamma;
    if (parts) gamma = sr_sum_parts(parts, n_parts, sh).x;
    else gamma = sc->gd[0];
    if (threadIdx.x != 0) return;
    const double normr = sqrt(gamma);
    const int run = (1 < max_iter) && normr > tol;
    sc->tol = tol;
    sc->max_iter = max_iter;
    sc->sr_k[0] = 1;
    sc->sr_gamma[0] = gamma;
    sc->sr_alpha[0] = 0.0;
    sc->run_q[0] = run;
    sc->run_q[1] = 0;
    sc->normr = normr;
    sc->niters = 0;
    sc->done = !run;
    sc->epoch = sc->epoch + 1;
    set_cond(cond, run);
}

// ------------------------------------------- persistent single-kernel solve
// For small single-GPU problems (configs[0], 20x30x10: everything fits in
// L2 and each kernel boundary costs more than the work), the whole HPCCG
// solve -- init and every iteration -- runs in ONE cooperative kernel: the
// phases are separated by a grid barrier (3 per iteration), every block sums
// the per-block partials itself in a fixed order (so all blocks hold
// bit-identical scalars and take identical loop decisions), and the loop
// control of A4/A11 is evaluated in registers.  Data written by other blocks
// inside the kernel (p, the partials) is read through L2 (ld.global.cg):
// L1 is not coherent within a launch.

struct PersistArgs {
    int64_t n, stride, plane;
    const double *val;
    const int *col;
    const double *b;
    double *x, *r, *p, *Ap;      // p: local-with-halo base
    double *part_rr, *part_pAp;  // gridDim.x partials each
    unsigned *bar;               // [0] arrivals, [32] generation (separate lines)
    CgScalars *sc;
    int max_iter;
    double tol;
};

// Grid-wide barrier for a cooperative launch (all blocks co-resident):
// arrival counter + generation flag, release/acquire at gpu scope.
__device__ __forceinline__ void grid_barrier(unsigned *bar, unsigned nblocks) {
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned *count = bar, *gen = bar + 32;
        unsigned g;
        asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(g) : "l"(gen) : "memory");
        __threadfence();
        unsigned t;
        asm volatile("atom.add.acq_rel.gpu.u32 %0, [%1], 1;" : "=r"(t) : "l"(count) : "memory");
        if (t == nblocks - 1) {
            asm volatile("st.relaxed.gpu.u32 [%0], %1;" ::"l"(count), "r"(0u) : "memory");
            asm volatile("st.release.gpu.u32 [%0], %1;" ::"l"(gen), "r"(g + 1) : "memory");
        } else {
            unsigned cur;
            do {
                asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(cur) : "l"(gen) : "memory");
            } while (cur == g);
        }
        __threadfence();
    }
    __syncthreads();
}

// Sum of the gridDim.x partials in a fixed order; identical in every block.
__device__ __forceinline__ double sum_partials(const double *part, double *sh) {
    double s = 0.0;
    for (unsigned i = threadIdx.x; i < gridDim.x; i += kBlock) s += __ldcg(part + i);
    __syncthreads();
    s = block_reduce<false>(s, sh);
    if (threadIdx.x == 0) sh[31] = s;
    __syncthreads();
    s = sh[31];
    __syncthreads();
    return s;
}

__device__ __forceinline__ double block_partial(double v, double *sh) {
    v = block_reduce<false>(v, sh);  // valid in warp 0
    __syncthreads();
    return v;
}

// kCluster: the whole grid is ONE thread-block cluster (<= 16 CTAs) and the
// phases are separated by the hardware cluster barrier (~380 cycles on
// Blackwell, and it invalidates L1) instead of the global-atomic grid barrier.
template <bool kCluster>
__device__ __forceinline__ void phase_barrier(unsigned *bar, unsigned nb) {
    if (kCluster) cooperative_groups::this_cluster().sync();
    else grid_barrier(bar, nb);
}

template <bool kCluster>
__global__ void __launch_bounds__(kBlock, 1) cg_persistent_kernel(PersistArgs a) {
    __shared__ double sh[32];
    const int64_t tid = gtid(), nth = gnth();
    const unsigned nb = gridDim.x;
    double *po = a.p + a.plane;
    auto spmv_row = [&](int64_t i) {
        double s = 0.0;
#pragma unroll 9
        for (int k = 0; k < kSlots; ++k)
            s = fma(__ldg(a.val + k * a.stride + i), __ldcg(a.p + __ldg(a.col + k * a.stride + i)), s);
        return s;
    };
    // ---- init (a.7): p = x; Ap = A p; r = b - Ap; rtrans = r.r
    for (int64_t i = tid; i < a.n; i += nth) po[i] = a.x[i];
    phase_barrier<kCluster>(a.bar, nb);
    double acc = 0.0;
    for (int64_t i = tid; i < a.n; i += nth) {
        const double ap = spmv_row(i);
        const double rv = fma(-1.0, ap, a.b[i]);
        a.r[i] = rv;
        acc = fma(rv, rv, acc);
    }
    acc = block_partial(acc, sh);
    if (threadIdx.x == 0) a.part_rr[blockIdx.x] = acc;
    phase_barrier<kCluster>(a.bar, nb);
    double rr = sum_partials(a.part_rr, sh);
    double rtrans = rr, normr = sqrt(rtrans);
    int niters = 0;
    // ---- HPCCG loop (a.8, A4 lag, A11 guard)
    for (int k = 1; k < a.max_iter && normr > a.tol; ++k) {
        double beta = 0.0;
        if (k > 1) {
            const double old = rtrans;
            rtrans = rr;
            beta = rtrans / old;
        }
        for (int64_t i = tid; i < a.n; i += nth) po[i] = (k == 1) ? a.r[i] : fma(beta, po[i], a.r[i]);
        normr = sqrt(rtrans);
        phase_barrier<kCluster>(a.bar, nb);
        double d = 0.0;
        for (int64_t i = tid; i < a.n; i += nth) {
            const double ap = spmv_row(i);
            a.Ap[i] = ap;
            d = fma(ap, po[i], d);
        }
        d = block_partial(d, sh);
        if (threadIdx.x == 0) a.part_pAp[blockIdx.x] = d;
        phase_barrier<kCluster>(a.bar, nb);
        const double pAp = sum_partials(a.part_pAp, sh);
        const bool stop = (rtrans == 0.0) || (pAp == 0.0);
        const double alpha = stop ? 0.0 : rtrans / pAp;
        acc = 0.0;
        for (int64_t i = tid; i < a.n; i += nth) {
            a.x[i] = fma(alpha, po[i], a.x[i]);
            const double rv = fma(-alpha, a.Ap[i], a.r[i]);
            a.r[i] = rv;
            acc = fma(rv, rv, acc);
        }
        acc = block_partial(acc, sh);
        if (threadIdx.x == 0) a.part_rr[blockIdx.x] = acc;
        phase_barrier<kCluster>(a.bar, nb);
        rr = sum_partials(a.part_rr, sh);
        niters = k;
        if (stop) break;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        a.sc->niters = niters;
        a.sc->normr = normr;
        a.sc->rr_cur = rr;
        a.sc->rr_prev = rtrans;
        a.sc->done = 1;
    }
}

// ----------------------------------- on-chip solve (tiny single-GPU problems)
// The whole problem lives in the shared memory of ONE thread-block cluster
// (<= 16 CTAs, 227 KB each): CTA c owns rows [c R, (c+1) R) -- its ELL slice,
// b, x, r, p, Ap -- loaded once per solve.  The stencil gathers read p from
// the owning CTA's shared memory (distributed shared memory when it is a
// neighbour CTA), every reduction is 16 per-CTA partials read by every CTA in
// rank order, and the phases are separated by the hardware cluster barrier.
// Same HPCCG loop (A4, A11) as every other path; per-row FMA chain as A8.
struct SmemArgs {
    int64_t n, stride, plane;
    int R;  // rows per CTA
    int nx, dia;  // dia: DIA-27 reading (HPCCG_OPT_SPMV_FORMAT 1) -- no column slice in smem (kDia)
    const double *val;
    const int *col;
    const double *b;
    double *x;  // in: initial guess, out: iterate
    CgScalars *sc;
    int max_iter;
    double tol;
    int H;      // > 0: the gathered vector is kept with H halo rows each side in every
                // CTA's own shared memory (refreshed once per SpMV by coalesced reads of
                // the owners' rows), so the 27 gathers of a row are local; 0: each
                // gather reads the owner CTA's shared memory (DSMEM)
};

// Block sum of two values over NT threads in a fixed order (butterfly per
// warp, then warp 0 over the per-warp values); valid in warp 0.
template <int NT>
__device__ __forceinline__ double2 blk_sum2(double u, double v, double *sh /*[64]*/) {
    constexpr int W = NT / 32;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    __syncwarp();
    u = warp_sum(u);
    v = warp_sum(v);
    if (lane == 0) {
        sh[warp] = u;
        sh[32 + warp] = v;
    }
    __syncwarp();
    __syncthreads();
    if (warp == 0) {
        u = warp_sum(lane < W ? sh[lane] : 0.0);
        v = warp_sum(lane < W ? sh[32 + lane] : 0.0);
    }
    return make_double2(u, v);
}

// Cluster-wide sums of (u, v): per-CTA block sums, one cluster barrier, then
// lanes 0..C-1 of warp 0 fetch the C partials in parallel (one DSMEM round
// trip) and a fixed butterfly: bit-identical sums in every CTA.  `mine` is
// this CTA's partial slot (2 doubles); the next write to it is separated from
// these reads by at least one more cluster barrier (callers' phase structure).
template <int NT>
__device__ __forceinline__ double2 cluster_sum2(double *mine, double u, double v, double *sh) {
    namespace cgx = cooperative_groups;
    auto cl = cgx::this_cluster();
    const double2 t = blk_sum2<NT>(u, v, sh);
    if (threadIdx.x == 0) {
        mine[0] = t.x;
        mine[1] = t.y;
    }
    cl.sync();
    if (threadIdx.x < 32) {
        const unsigned c = threadIdx.x;
        double qu = 0.0, qv = 0.0;
        if (c < cl.num_blocks()) {
            const double *m = cl.map_shared_rank(mine, c);
            qu = m[0];
            qv = m[1];
        }
        qu = warp_sum(qu);
        qv = warp_sum(qv);
        if (threadIdx.x == 0) {
            sh[64] = qu;
            sh[65] = qv;
        }
    }
    __syncthreads();
    // (no trailing barrier: sh[64..65] is written again only by warp 0 of the next
    // call after that call's block barrier, which every reader has passed)
    return make_double2(sh[64], sh[65]);
}

// ----------------------------------- on-chip solve (tiny single-GPU problems)
// The whole problem lives in the shared memory of ONE thread-block cluster
// (<= 16 CTAs, 227 KB each): CTA c owns rows [c R, (c+1) R) -- its ELL slice,
// b and the CG vectors -- loaded once per solve.  The stencil gathers read the
// gathered vector from the owning CTA's shared memory (distributed shared
// memory when it is a neighbour CTA), every reduction is C per-CTA partials
// read by every CTA in rank order, and the phases are separated by the
// hardware cluster barrier.  NT threads per CTA (512 when R > 256, so each
// thread's rows are gathered in one trip).
//   kSR = false: HPCCG's CG (A4, A11), 3 cluster barriers per iteration;
//   kSR = true:  the single-reduction CG of f2 (oracle_cg_sr), 2 per iteration.
// Per-row FMA chain as A8.
// kHalo (HPCCG_OPT_SMEM_HALO): a.H > 0 halo rows, gathers from the local copy
template <int NT, bool kSR, bool kDia = false, bool kHalo = false>
__global__ void __launch_bounds__(NT, 1) cg_smem_cluster_kernel(SmemArgs a) {
    namespace cgx = cooperative_groups;
    auto cl = cgx::this_cluster();
    extern __shared__ double smem[];
    __shared__ double sh[66];
    __shared__ double part_a[2], part_b[2];
    const int R = a.R;
    const unsigned me = cl.block_rank();
    const int Hh = kHalo ? a.H : 0;             // halo rows of the gathered vector (0: DSMEM gathers)
    double *sval = smem;                        // [27][R]
    double *sb = sval + (size_t)kSlots * R;     // [R] each
    // the gathered vector (SR: r, HPCCG: p) gets Hh halo rows on each side
    double *sx = sb + R, *sr = sx + R + (kSR ? Hh : 0);
    double *sp = sr + R + (kSR ? Hh : Hh);      // (SR: after r's upper halo; HPCCG: after p's lower halo)
    double *sq = sp + R + (kSR ? 0 : Hh);       // sq: Ap (HPCCG) / w (SR)
    double *ss = sq + R;                        // SR: s = A p recurrence
    int *scol = reinterpret_cast<int *>(ss + (kSR ? R : 0));  // [27][R]
    const int64_t row0 = (int64_t)me * R;
    const int64_t rem = a.n - row0;
    const int nr = rem <= 0 ? 0 : (int)(rem < R ? rem : R);
    // matrix rows into shared memory: all 27 slots' loads of a row issued before
    // any store (one HBM round trip per trip instead of one per slot)
    for (int i = threadIdx.x; i < nr; i += NT) {
        double v[kSlots];
        int cidx[kSlots];
#pragma unroll
        for (int k = 0; k < kSlots; ++k) {
            v[k] = __ldcs(a.val + k * a.stride + row0 + i);
            cidx[k] = kDia ? 0 : __ldcs(a.col + k * a.stride + row0 + i);
        }
        const double bv = a.b[row0 + i], xv = a.x[row0 + i];
#pragma unroll
        for (int k = 0; k < kSlots; ++k) {
            sval[k * R + i] = v[k];
            if (!kDia) scol[k * R + i] = cidx[k];
        }
        sb[i] = bv;
        sx[i] = xv;
    }
    __syncthreads();
    const int plane32 = (int)a.plane;
    // y_i = sum_k val * g[col], g = the gathered vector, read from its owner CTA
    auto spmv_row = [&](const double *g, int i) {
        double pv[kSlots];
        const int own = (int)row0 + i;
#pragma unroll
        for (int k = 0; k < kSlots; ++k) {  // all 27 gathers issued before the FMA chain
            // global row of the column (< 2^31); DIA: from the stencil offset, padding -> own
            const int c = kDia ? (sval[k * R + i] != 0.0
                                       ? own + (k / 9 - 1) * plane32 + ((k / 3) % 3 - 1) * a.nx + (k % 3 - 1)
                                       : own)
                                : scol[k * R + i] - plane32;
            if (kHalo) {  // local copy: own rows at g[0, R), halo at g[-Hh, 0) and g[R, R + Hh)
                pv[k] = g[c - (int)row0];
            } else {
                const unsigned owner = (unsigned)c / (unsigned)R;
                const int off = c - (int)owner * R;
                pv[k] = *cl.map_shared_rank(g + off, owner);
            }
        }
        double s = 0.0;
#pragma unroll
        for (int k = 0; k < kSlots; ++k) s = fma(sval[k * R + i], pv[k], s);
        return s;
    };
    // kHalo: a new value v of own row i of the gathered vector g is also stored
    // into the halo copy of every other CTA whose window [c R - Hh, c R + R + Hh)
    // holds that row (distributed shared memory stores, no round trip); the
    // cluster barrier that follows makes them visible before any gather.  The
    // receivers read those copies only between that barrier and the next one.
    const int nct = (int)cl.num_blocks();
    auto put = [&](double *g, int i, double v) {
        g[i] = v;
        if (!kHalo) return;
        const int64_t gr = row0 + i;
        const int c_hi = min(nct - 1, (int)((gr + Hh) / R));
        for (int c = max(0, (int)((gr - Hh - R) / R)); c <= c_hi; ++c) {
            const int64_t off = gr - (int64_t)c * R;  // the row in CTA c's window
            if (c == (int)me || off < -Hh || off >= R + Hh) continue;
            *cl.map_shared_rank(g + off, (unsigned)c) = v;
        }
    };
    int niters = 0;
    double normr, rr_out, rr_prev_out;
    if (!kSR) {
        // ---- init (a.7): p = x; Ap = A p; r = b - Ap; rtrans = r.r
        for (int i = threadIdx.x; i < nr; i += NT) put(sp, i, sx[i]);
        cl.sync();
        double acc = 0.0;
        for (int i = threadIdx.x; i < nr; i += NT) {
            const double rv = fma(-1.0, spmv_row(sp, i), sb[i]);
            sr[i] = rv;
            acc = fma(rv, rv, acc);
        }
        double rr = cluster_sum2<NT>(part_b, acc, 0.0, sh).x;
        double rtrans = rr;
        normr = sqrt(rtrans);
        for (int k = 1; k < a.max_iter && normr > a.tol; ++k) {
            double beta = 0.0;
            if (k > 1) {
                const double old = rtrans;
                rtrans = rr;
                beta = rtrans / old;
            }
            // every CTA has finished reading the previous p (cluster_sum2's barrier)
            for (int i = threadIdx.x; i < nr; i += NT) put(sp, i, (k == 1) ? sr[i] : fma(beta, sp[i], sr[i]));
            normr = sqrt(rtrans);
            cl.sync();
            double d = 0.0;
            for (int i = threadIdx.x; i < nr; i += NT) {
                const double ap = spmv_row(sp, i);
                sq[i] = ap;
                d = fma(ap, sp[i], d);
            }
            const double pAp = cluster_sum2<NT>(part_a, d, 0.0, sh).x;
            const bool stop = (rtrans == 0.0) || (pAp == 0.0);
            const double alpha = stop ? 0.0 : rtrans / pAp;
            acc = 0.0;
            for (int i = threadIdx.x; i < nr; i += NT) {
                sx[i] = fma(alpha, sp[i], sx[i]);
                const double rv = fma(-alpha, sq[i], sr[i]);
                sr[i] = rv;
                acc = fma(rv, rv, acc);
            }
            rr = cluster_sum2<NT>(part_b, acc, 0.0, sh).x;
            niters = k;
            if (stop) break;
        }
        rr_out = rr;
        rr_prev_out = rtrans;
    } else {
        // ---- init: r = b - A x0 (x0 gathered from sr), w = A r, (gamma, delta)
        for (int i = threadIdx.x; i < nr; i += NT) put(sr, i, sx[i]);
        cl.sync();
        for (int i = threadIdx.x; i < nr; i += NT) sq[i] = fma(-1.0, spmv_row(sr, i), sb[i]);
        cl.sync();  // every CTA has finished gathering x0 from sr
        for (int i = threadIdx.x; i < nr; i += NT) put(sr, i, sq[i]);
        cl.sync();
        double g = 0.0, dl = 0.0;
        for (int i = threadIdx.x; i < nr; i += NT) {
            const double w = spmv_row(sr, i);
            sq[i] = w;
            g = fma(sr[i], sr[i], g);
            dl = fma(w, sr[i], dl);
        }
        double2 gd = cluster_sum2<NT>(part_a, g, dl, sh);
        double gamma = gd.x, delta = gd.y, gamma_old = 0.0, alpha_old = 0.0;
        normr = sqrt(gamma);
        for (int k = 1; k < a.max_iter && normr > a.tol; ++k) {
            const bool first = (k == 1);
            const double beta = first ? 0.0 : __ddiv_rn(gamma, gamma_old);
            const double den = first ? delta : __dsub_rn(delta, __ddiv_rn(__dmul_rn(beta, gamma), alpha_old));
            const bool stop = (gamma == 0.0) || (den == 0.0);  // A11
            const double alpha = stop ? 0.0 : __ddiv_rn(gamma, den);
            normr = sqrt(gamma);
            // every CTA has finished gathering r (cluster_sum2's barrier)
            for (int i = threadIdx.x; i < nr; i += NT) {
                const double pv = first ? sr[i] : fma(beta, sp[i], sr[i]);
                const double sv = first ? sq[i] : fma(beta, ss[i], sq[i]);
                sp[i] = pv;
                ss[i] = sv;
                sx[i] = fma(alpha, pv, sx[i]);
                put(sr, i, fma(-alpha, sv, sr[i]));
            }
            niters = k;
            // the next iteration would not run (A4, A11): skip its SpMV
            if (stop || !(k + 1 < a.max_iter && normr > a.tol)) break;
            cl.sync();
            g = 0.0;
            dl = 0.0;
            for (int i = threadIdx.x; i < nr; i += NT) {
                const double w = spmv_row(sr, i);
                sq[i] = w;
                g = fma(sr[i], sr[i], g);
                dl = fma(w, sr[i], dl);
            }
            gd = cluster_sum2<NT>((k & 1) ? part_b : part_a, g, dl, sh);
            gamma_old = gamma;
            gamma = gd.x;
            delta = gd.y;
            alpha_old = alpha;
        }
        rr_out = gamma;
        rr_prev_out = gamma_old;
    }
    for (int i = threadIdx.x; i < nr; i += NT) a.x[row0 + i] = sx[i];
    if (me == 0 && threadIdx.x == 0) {
        a.sc->niters = niters;
        a.sc->normr = normr;
        a.sc->rr_cur = rr_out;
        a.sc->rr_prev = rr_prev_out;
        a.sc->done = 1;
    }
    cl.sync();  // no CTA leaves while its shared memory may still be read
}

// Loopback allreduce: fixed rank-order sum (or max) of one scalar of every
// slab, written back to every slab (deterministic, identical on all slabs).
__global__ void slab_allreduce_kernel(const double *const *src, double *const *dst,
                                      int nslabs, int is_max, int count) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    for (int c = 0; c < count; ++c) {
        double s = src[0][c];
        for (int r = 1; r < nslabs; ++r) s = is_max ? fmax(s, src[r][c]) : s + src[r][c];
        for (int r = 0; r < nslabs; ++r) dst[r][c] = s;
    }
}

// ------------------------------- peer-memory z-slab exchange (HALO_PEER)
// The multi-slab iteration's two collectives done by our own kernels over
// peer memory (NVLink P2P on a multi-GPU node; sibling slabs' buffers in
// loopback): the halo exchange is a PUSH -- each slab stores its first and
// last owned planes straight into its neighbours' halo planes and then
// signals them -- and each scalar allreduce is a POST of the local value into
// slot [rank] of every peer followed by a COLLECT that waits for the P slots
// and sums them in rank order (deterministic, bit-identical on every rank, and
// bit-identical to the loopback allreduce kernel).  Counters advance in
// lockstep on every slab (every slab runs every exchange and allreduce), so a
// flag / tag is the count of the operation it completes.  Two slot sets
// (count parity) suffice: a rank cannot post allreduce m + 2 before every rank
// has collected m (it needs all ranks' m + 1 posts, made after their collect
// of m).  A push overwrites the neighbour's halo with no handshake, so the
// caller must separate consecutive exchanges by an allreduce (a rank posts
// only after its boundary SpMV has read the previous halo): the CG iterations
// do by construction, and the f2 init adds one between its two exchanges.
// Memory model: pushes / posts, then fence.sc.sys, then a st.release.sys
// of the flag / tag; waits are ld.acquire.sys spins, bounded by a %globaltimer
// timeout that records an error instead of hanging the GPU.

// a.2 push: my first owned plane -> rank-1's upper halo, my last owned plane
// -> rank+1's lower halo (x = local-with-halo base); the last block signals.
__global__ void __launch_bounds__(kBlock) halo_push_kernel(const PeerTab *t, const double *x, int64_t n,
                                                         int64_t plane) {
    const int64_t tid = gtid(), nth = gnth();
    double *lo = t->halo_to_lo, *hi = t->halo_to_hi;
    for (int64_t i = tid; i < 2 * plane; i += nth) {
        if (i < plane) {
            if (lo) lo[i] = x[plane + i];
        } else if (hi) {
            hi[i - plane] = x[n + (i - plane)];
        }
    }
    __shared__ int last;
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence_system();  // my pushes before the ticket (and so before the flag)
        const unsigned tk = atomicAdd(&t->mine->push_ticket, 1u);
        last = (tk == gridDim.x - 1);
    }
    __syncthreads();
    if (!last || threadIdx.x != 0) return;
    __threadfence_system();
    t->mine->push_ticket = 0u;
    const unsigned long long c = t->mine->push_count + 1;
    t->mine->push_count = c;
    if (t->lo) st_release_sys(&t->lo->flag_from_hi, c);
    if (t->hi) st_release_sys(&t->hi->flag_from_lo, c);
}

// a.2 wait: both neighbours have pushed this exchange (one thread).
__global__ void halo_wait_kernel(const PeerTab *t) {
    if (threadIdx.x != 0) return;
    PeerSync *m = t->mine;
    const unsigned long long target = m->recv_count + 1;
    if (t->rank > 0 && !spin_until(&m->flag_from_lo, target, m, PEER_WAIT_HALO_LO, t->rank - 1)) return;
    if (t->rank < t->nranks - 1 &&
        !spin_until(&m->flag_from_hi, target, m, PEER_WAIT_HALO_HI, t->rank + 1))
        return;
    m->recv_count = target;
}

// a.4/a.5 allreduce over peer memory of `count` (<= 2) doubles: post (my
// values into slot [rank] of every rank, then the tag) and / or collect (wait
// for the P tags, sum in rank order -- or max -- into dst).  One warp.
__global__ void peer_allreduce_kernel(const PeerTab *t, const double *src, double *dst, int count,
                                      int is_max, int post, int collect) {
    PeerSync *m = t->mine;
    const int P = t->nranks, lane = threadIdx.x;
    if (post) {
        const unsigned long long c = m->ar_posted + 1;
        const int q = (int)(c & 1);
        for (int r = lane; r < P; r += 32) {
            PeerSync *dstp = t->all[r];
            for (int j = 0; j < count; ++j) dstp->ar_val[q][t->rank][j] = src[j];
            __threadfence_system();
            st_release_sys(&dstp->ar_tag[q][t->rank], c);
        }
        __syncwarp();
        if (lane == 0) m->ar_posted = c;
    }
    if (collect) {
        const unsigned long long c = m->ar_count + 1;
        const int q = (int)(c & 1);
        for (int r = lane; r < P; r += 32)
            if (!spin_until(&m->ar_tag[q][r], c, m, PEER_WAIT_ALLREDUCE, r)) break;
        __syncwarp();
        if (lane == 0) {
            __threadfence();
            for (int j = 0; j < count; ++j) {
                double s = m->ar_val[q][0][j];
                for (int r = 1; r < P; ++r) s = is_max ? fmax(s, m->ar_val[q][r][j]) : s + m->ar_val[q][r][j];
                dst[j] = s;
            }
            m->ar_count = c;
        }
    }
}

// ---------------------------------------------------------- a.10 BLAS-1

// w = alpha x + beta y, canonical forms (A10).  form: 0 alpha==1, 1 beta==1,
// 2 general.  24n B.  kU 16-B units per thread per trip, all loads issued
// before the stores (plain loads: evict-first ones measured slower here).
template <bool kVec, int kForm, int kU = 2>
__global__ void __launch_bounds__(kBlock) waxpby_kernel(int64_t n, double alpha, const double *x,
                                                       double beta, const double *y, double *w) {
    const int64_t tid = gtid(), nth = gnth();
    auto op = [alpha, beta](double xv, double yv) {
        if (kForm == 0) return fma(beta, yv, xv);
        if (kForm == 1) return fma(alpha, xv, yv);
        return fma(alpha, xv, beta * yv);
    };
    if (kVec) {
        const int64_t nv = n >> 1;
        const double2 *x2 = reinterpret_cast<const double2 *>(x);
        const double2 *y2 = reinterpret_cast<const double2 *>(y);
        double2 *w2 = reinterpret_cast<double2 *>(w);
        for (int64_t i = tid; i < nv; i += kU * nth) {
            double2 xa[kU], ya[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int64_t j = i + u * nth;
                if (j < nv) {
                    xa[u] = x2[j];
                    ya[u] = y2[j];
                }
            }
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int64_t j = i + u * nth;
                if (j < nv) w2[j] = make_double2(op(xa[u].x, ya[u].x), op(xa[u].y, ya[u].y));
            }
        }
        if (tid == 0 && (n & 1)) w[n - 1] = op(x[n - 1], y[n - 1]);
    } else {
        for (int64_t i = tid; i < n; i += nth) w[i] = op(x[i], y[i]);
    }
}

// sum_i x_i y_i -> *out (deterministic: the element -> thread map and the
// per-thread order depend only on (n, grid, kU)).  16n B (8n for x.x).  kU
// 16-B units of x and y per thread per trip, all loads first, streamed.
template <bool kVec, int kU = 2>
__global__ void __launch_bounds__(kBlock) dot_kernel(int64_t n, const double *x, const double *y,
                                                    Reduction red, double *out) {
    const int64_t tid = gtid(), nth = gnth();
    double acc = 0.0;
    if (kVec) {
        const int64_t nv = n >> 1;
        const double2 *x2 = reinterpret_cast<const double2 *>(x);
        const double2 *y2 = reinterpret_cast<const double2 *>(y);
        double acc2 = 0.0;
        for (int64_t i = tid; i < nv; i += kU * nth) {
            double2 xa[kU], ya[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int64_t j = i + u * nth;
                xa[u] = make_double2(0.0, 0.0);   // zero-padded past nv
                ya[u] = make_double2(0.0, 0.0);
                if (j < nv) {
                    xa[u] = __ldcs(x2 + j);
                    ya[u] = __ldcs(y2 + j);
                }
            }
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                acc = fma(xa[u].x, ya[u].x, acc);
                acc2 = fma(xa[u].y, ya[u].y, acc2);
            }
        }
        acc += acc2;
        if (tid == 0 && (n & 1)) acc = fma(x[n - 1], y[n - 1], acc);
    } else {
        for (int64_t i = tid; i < n; i += nth) acc = fma(x[i], y[i], acc);
    }
    grid_reduce<false>(acc, red, blockIdx.x, gridDim.x, [out](double s) { *out = s; });
}

// ----------------------------------------------- f3: JACC 2-D AXPY / DOT
// JACC's multidimensional parallel_for / parallel_reduce over (M, N) on
// column-major arrays with leading dimension ld (Fig. 2; the CUDA
// back end uses 16x16 thread blocks, Fig. 6).  Here the blocks are
// 32 x 8: threadIdx.x walks the contiguous row index i, so a warp reads one
// 256-B segment of a column (coalesced); grid-stride in both dimensions.
constexpr int kB2x = 32, kB2y = 8;

template <int kForm>
__global__ void __launch_bounds__(kB2x *kB2y) waxpby2d_kernel(int64_t m, int64_t n, int64_t ld,
                                                              double alpha, const double *x,
                                                              double beta, const double *y,
                                                              double *w) {
    auto op = [alpha, beta](double xv, double yv) {
        if (kForm == 0) return fma(beta, yv, xv);
        if (kForm == 1) return fma(alpha, xv, yv);
        return fma(alpha, xv, beta * yv);
    };
    const int64_t si = (int64_t)gridDim.x * kB2x;
    for (int64_t j = (int64_t)blockIdx.y * kB2y + threadIdx.y; j < n; j += (int64_t)gridDim.y * kB2y)
        for (int64_t i0 = (int64_t)blockIdx.x * kB2x + threadIdx.x; i0 < m; i0 += 4 * si) {
            double xv[4], yv[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int64_t i = i0 + u * si;
                if (i < m) {
                    xv[u] = x[i + j * ld];
                    yv[u] = y[i + j * ld];
                }
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int64_t i = i0 + u * si;
                if (i < m) w[i + j * ld] = op(xv[u], yv[u]);
            }
        }
}

// launched with 1-D blocks of kB2x*kB2y threads (the reduction helpers index
// threads by threadIdx.x); (tx, ty) is the 32 x 8 tile position
__global__ void __launch_bounds__(kB2x *kB2y) dot2d_kernel(int64_t m, int64_t n, int64_t ld,
                                                           const double *x, const double *y,
                                                           Reduction red, double *out) {
    const int tx = threadIdx.x % kB2x, ty = threadIdx.x / kB2x;
    double acc = 0.0;
    const int64_t si = (int64_t)gridDim.x * kB2x;
    for (int64_t j = (int64_t)blockIdx.y * kB2y + ty; j < n; j += (int64_t)gridDim.y * kB2y)
        for (int64_t i0 = (int64_t)blockIdx.x * kB2x + tx; i0 < m; i0 += 4 * si) {
            double xv[4], yv[4];  // 4 independent loads per array in flight
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int64_t i = i0 + u * si;
                xv[u] = i < m ? __ldcs(x + i + j * ld) : 0.0;
                yv[u] = i < m ? __ldcs(y + i + j * ld) : 0.0;
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) acc = fma(xv[u], yv[u], acc);
        }
    // flatten the 2-D block into the 1-D reduction helpers (256 threads)
    grid_reduce<false>(acc, red, blockIdx.y * gridDim.x + blockIdx.x, gridDim.x * gridDim.y,
                       [out](double v) { *out = v; });
}

// a.9: max_i |x_i - xe_i| -> *out
__global__ void __launch_bounds__(kBlock) maxabsdiff_kernel(int64_t n, const double *x,
                                                           const double *xe, Reduction red,
                                                           double *out) {
    const int64_t tid = gtid(), nth = gnth();
    double m = 0.0;
    for (int64_t i = tid; i < n; i += nth) m = fmax(m, fabs(x[i] - xe[i]));
    grid_reduce<true>(m, red, blockIdx.x, gridDim.x, [out](double s) { *out = s; });
}

// p = x for the owned part (init, waxpby(1, x, 0, x, p) = x exactly).
__global__ void __launch_bounds__(kBlock) copy_kernel(int64_t n, const double *src, double *dst) {
    const int64_t tid = gtid(), nth = gnth();
    for (int64_t i = tid; i < n; i += nth) dst[i] = src[i];
}

}  // namespace hpccg
