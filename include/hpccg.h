/*
 * hpccg.h -- C ABI of the B200-native HPCCG conjugate-gradient hot path.
 *
 * The library (libhpccg.so, built from paper_conf_sc_valero_laragmtv24_b200/
 * csrc/) runs every step of the path in hand-written sm_100a CUDA kernels:
 * on-device problem generation, the 27-point SpMV, the ddot reductions and
 * the waxpby updates, with the dots fused into the updates, and a z-slab
 * ("chimney") decomposition across GPUs with NCCL halo-plane exchange and one
 * scalar allreduce per dot (BASELINE.json north_star).
 *
 * Citations: "P:Lnnn" = line of the paper text (Valero-Lara et al., "JACC",
 * SC'24 workshops, PAPER.md); "north_star" = BASELINE.json; "A<k>" = reading
 * k in DESIGN.md (sec. Readings).  HPCCG = the Mantevo HPCCG 1.0 benchmark the
 * paper names (P:L7), whose call signatures
 * generate_matrix / HPC_sparsemv / ddot / waxpby / HPCCG this ABI follows.
 *
 * Conventions (all functions):
 *  - Return HPCCG_OK (0) or a negative HPCCG_E* code; never abort or throw.
 *    hpccg_strerror(code) names the code, hpccg_last_error() gives the
 *    detail message of the calling thread's last failure.
 *  - Every call is host-synchronous on return: device work it enqueued has
 *    completed (JACC's constructs are synchronous).
 *  - SPMD: with nranks > 1 every rank calls every function collectively, in
 *    the same order, like HPCCG-MPI.
 *  - "device" pointers are CUDA device pointers on the context's device
 *    (e.g. torch.empty(..., device='cuda').data_ptr()); the caller owns them.
 *    Objects returned through ** out-parameters are library-owned until the
 *    matching hpccg_free / hpccg_finalize.
 *  - fp64 everywhere ("All computations are double-precision").
 *  - Loopback contexts (hpccg_init_loopback) host all nranks slabs in ONE
 *    process on ONE device, for testing the decomposition without NCCL.  In
 *    that mode every "local vector" argument is the concatenation, in rank
 *    order, of the nranks per-rank local vectors, and every length n is the
 *    per-rank length.
 *  - One context per host thread (thread-compatible, not thread-safe).
 */
#ifndef HPCCG_H
#define HPCCG_H

#include <stdint.h>

#if defined(__GNUC__)
#define HPCCG_API __attribute__((visibility("default")))
#else
#define HPCCG_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

#define HPCCG_OK 0
#define HPCCG_EINVAL (-1)   /* bad argument (sizes < 1, n > local length, NULL) */
#define HPCCG_ENOMEM (-2)   /* device or host allocation failed */
#define HPCCG_ECUDA (-3)    /* a CUDA runtime call or kernel launch failed */
#define HPCCG_ENCCL (-4)    /* an NCCL call failed (comm aborted) */
#define HPCCG_ENOTSUP (-5)  /* not available in this build / configuration */

#define HPCCG_UNIQUE_ID_BYTES 128

/* which vector hpccg_vec / hpccg_set_vec / hpccg_get_vec address */
#define HPCCG_VEC_X 0       /* iterate / initial guess, nrow_local */
#define HPCCG_VEC_B 1       /* right-hand side b = A.1, nrow_local */
#define HPCCG_VEC_XEXACT 2  /* exact solution (all ones), nrow_local */

/* hpccg_set_option keys */
#define HPCCG_OPT_GRAPH 0   /* 1 (default): replay each CG iteration as a CUDA graph */
#define HPCCG_OPT_POLL 1    /* iterations between host polls of the device stop flag
                               when tol > 0 (default 8); 0 = never poll */
#define HPCCG_OPT_TIMING 2  /* 1: CUDA-event time every phase of every iteration into
                               hpccg_get_stats / times[] (disables the graph); default 0 */
#define HPCCG_OPT_SPMV_MINB 3 /* SpMV register budget: min resident 256-thread blocks per
                               SM (1..4; 0 = tuned default) -- a tuning knob */
#define HPCCG_OPT_WHILE 4   /* 1 (default): with GRAPH, run the whole solve as one graph
                               with a device-driven conditional WHILE node (single GPU /
                               loopback); 0: replay a per-iteration graph with host polls */
#define HPCCG_OPT_L2_PERSIST 5 /* 1 (default): during hpccg_solve, mark the CG vectors
                               (r, x, Ap, p) L2-persisting via an access-policy window on
                               the stream (restored afterwards); 0: off */
#define HPCCG_OPT_SPMV_ROWS 7 /* SpMV rows per thread: 2 (default; needs even n and plane,
                               else 1 is used), 1 */
#define HPCCG_OPT_VEC_UNROLL 8 /* CG vector kernels: 16-B units per thread per trip with
                               all loads in flight: 1, 2 or 4 (default 4) */
#define HPCCG_OPT_PERSISTENT 9 /* single GPU: run the whole solve as ONE cooperative kernel
                               (grid barriers between phases): 0 never, 1 (default) auto
                               (HPCCG_OPT_PERSIST_ROWS), 2 always */
#define HPCCG_OPT_PERSIST_ROWS 10 /* threshold for HPCCG_OPT_PERSISTENT = 1: -1 (default) only
                               when the whole problem fits the on-chip (shared-memory) solve
                               (the while-graph is faster above that); k >= 0:
                               when nrow_local <= k */
#define HPCCG_OPT_SMEM_SOLVE 13 /* 1 (default): a persistent solve whose rows fit in the
                               shared memory of one 16-CTA cluster keeps the whole problem on
                               chip (distributed shared memory gathers): ~9.9k rows with the ELL
                               slice (HPCCG_OPT_SPMV_FORMAT 0), ~14k rows under format 1 (no column
                               slice); 0: off */
#define HPCCG_OPT_TRACE 14  /* k > 0: record, for the first k iterations, each CG kernel's
                               first-block start and last-block end on the device clock
                               (%globaltimer; works inside graphs); read with
                               hpccg_get_trace.  0 (default): off */
#define HPCCG_OPT_CG_VARIANT 16 /* 0 (default): HPCCG's CG (SpMV + p.Ap, x/r update + r.r,
                               p update; two reductions per iteration).  1: single-reduction
                               (Chronopoulos-Gear) CG: same iterates in exact
                               arithmetic, two kernels per iteration (one fused update of
                               p, s = A p, x, r; the SpMV w = A r with r.r and w.r in its
                               epilogue) and ONE allreduce of two values; needs 8n more bytes
                               (s), small problems use the graph path instead of the
                               persistent kernel.  Rounding differs: niters +-1 */
#define HPCCG_OPT_FINISHER_FREE 17 /* 1 (default): single GPU, HPCCG variant: no grid-wide
                               finisher in any CG kernel -- the x/r update writes per-block
                               r.r partials that every block of the next p update sums in
                               the finisher's fixed order (identical bits), and takes the
                               loop decision itself; 0: the update's last block finishes
                               r.r and the loop control */
#define HPCCG_OPT_SMEM_THREADS 18 /* threads per CTA of the shared-memory-resident solve:
                               0 (default) auto (512 when a CTA holds > 256 rows), 256, 512 */
#define HPCCG_OPT_HALO_PEER 19 /* multi-slab: 1 = the halo exchange and the scalar allreduces
                               run as this library's own kernels over PEER MEMORY -- each slab
                               pushes its boundary planes straight into its neighbours' halo
                               planes and signals them (flag + system-scope release), and each
                               allreduce posts the local value into slot [rank] of every peer and
                               sums the P slots in rank order -- instead of NCCL send/recv /
                               ncclAllReduce (or the loopback copies).  NCCL contexts map the
                               peers' buffers with CUDA IPC (collective: every rank sets it);
                               loopback contexts use the sibling slabs.  0 (default): off.
                               2: the same exchange and allreduces FUSED into the CG kernels
                               (HPCCG variant; no push / wait / allreduce kernels, no comm
                               stream): the p update stores its boundary planes into the
                               neighbours' halos as it computes them and raises their flags,
                               the SpMV's boundary row blocks wait for the flags and its last
                               block posts p.Ap to every rank, every block of the x/r update
                               collects the P posts (rank order) and its last block posts r.r,
                               which every block of the next p update collects -- 3 kernels
                               per iteration; needs even nx*ny and n, else behaves as 1.
                               Bit-identical to the loopback reduction order.  Waits time out
                               after HPCCG_OPT_PEER_TIMEOUT_MS with HPCCG_ECUDA instead of
                               hanging; hpccg_last_error() names the rank that gave up, what it
                               waited for (halo plane / allreduce post) and the peer it waited
                               on.  The record is sticky: a slab that timed out has lost step
                               with its peers, so every later hpccg_solve of that problem
                               returns HPCCG_ECUDA at once (recreate the problem).  The value
                               is range-checked before any peer mapping is attempted. */
#define HPCCG_OPT_DEFER_X 23 /* finisher-free HPCCG loop (single slab, or z-slabs with
                               HALO_PEER 2): 1 defers x += alpha p of iteration k
                               into the p update of iteration k + 1 (which reads p_k anyway;
                               cg_xfix_kernel applies the last one after the loop), so the
                               x/r update moves 24n instead of 48n B and the p update 40n
                               instead of 24n: 80n + 12 nnz B per iteration instead of 88n.
                               Bitwise the same results (the same FMA on the same operands);
                               0: x updated in the x/r update.  m = 2..8 (single slab only;
                               z-slabs fall back to 1): deferred over a ring of m + 1 p buffers
                               -- p_k is written to slot k % (m + 1) (slot 0 = the problem's p
                               buffer, the SpMV gathers from the slot of iteration k) and every
                               m-th p update applies x = fma(alpha_j, p_j, x) for the m
                               directions since the last one, in ascending j; the pending ones
                               run after the loop (cg_xfix_ring_kernel).  On z-slabs (HALO_PEER 2)
                               the p update pushes p_k's boundary planes into slot k % (m + 1) of
                               the neighbours' rings: a ring is exchanged only if it exists when the
                               peer tables are built (auto: allocated at generate; explicit m on
                               one-slab-per-process contexts: set it before HALO_PEER / the peer
                               export), else z-slabs run m = 1; every rank must use the same value
                               (the neighbours' slots are addressed by k % (m + 1)).  Per m iterations x
                               is read and written once and m - 1 old p's re-read: 12 nnz +
                               (72 + 8/m) n B per iteration, the writes drop from 2 to 1 + 1/m
                               per row.  Bitwise the same results.  Device memory: m extra
                               p-sized buffers per slab (allocated when the option is set, or at
                               generate time for auto).  The single-reduction CG (CG_VARIANT 1)
                               defers x over its own (not gathered) p vector the same way, any
                               context.  -1 (default): auto -- 8 when the CG
                               vectors exceed L2, 0 below (at 128^3 the vectors are L2-resident
                               and 0 is 0.4 % faster) */
#define HPCCG_OPT_FUSE_PSPMV 24 /* single slab, finisher-free loop: the p update and the
                               SpMV of an iteration as ONE pipelined kernel (cg_pspmv_kernel:
                               chunks of 512 rows taken in launch order; each block updates p
                               a fixed lead of chunks ahead and publishes it, then waits for
                               the <= 9 chunks its gathers read) -- p is gathered from L2
                               right after it is written: 12 nnz + 72n B per iteration with
                               the deferred x update (ncu at 256^3: 6.23 GB DRAM per launch,
                               p gathered from L2).  Bitwise the same results.  0 (default)
                               off -- measured no faster: the mixed read/write stream runs at
                               6.84 TB/s where the plain SpMV reaches 7.11, which eats the
                               8n B saved (256^3: 977 vs 978 us/iteration; 128^3 122 vs 115);
                               1 on, -1 auto (on when the CG vectors exceed L2) */
#define HPCCG_OPT_SPMV_TRIPS 26 /* single slab, finisher-free loop: 512-row trips per block of
                               the CG SpMV (spmv27x2_trips_kernel; one p.Ap partial per block),
                               so a slab with more than 4096 row blocks (256^3: 32768) needs no
                               1024-thread p.Ap finisher kernel -- the update blocks sum the
                               partials.  1 (default) off, 0 auto (the fewest trips that leave
                               <= 4096 partials), T > 1 explicit.  Same Ap bits; the p.Ap sum
                               takes another (fixed) tree.  Measured slower: 256^3 1066.7 (8
                               trips) vs 984.7 us/iteration, 512^3 8593 vs 8019 -- a block's
                               trips run back to back, so its loads drain between them */
#define HPCCG_OPT_PAP_CLUSTER 27 /* p.Ap finisher of a slab whose SpMV leaves more than 4096
                               partials (256^3: 32768): 0 one 1024-thread CTA, 1 one cluster of 8
                               CTAs reading the partials in parallel (distributed shared memory
                               for the 8 CTA sums).  Every mode of a problem uses the same one
                               (identical bits across modes); the two differ in the last bits.
                               Measured no faster (256^3 986.3 vs 986.0 us/iteration): default 0 */
#define HPCCG_OPT_SMEM_HALO 30 /* the on-chip (shared-memory cluster) solve: every CTA keeps the
                               gathered vector (p; r for the single-reduction CG) with the
                               stencil's reach (plane + nx + 1 rows) of halo on each side in its
                               own shared memory (every writer of an own row also stores it into
                               the windows of the CTAs that hold it, published by the cluster
                               barrier that follows), so the 27 gathers of a row are local
                               instead of distributed-shared-memory reads.  The same values in
                               the same order: bitwise the unhalo'd solve.  -1 (default) auto /
                               1: when the halo (16 (plane + nx + 1) B per CTA) fits next to the
                               rows; 0 off */
#define HPCCG_OPT_SPMV_CLUSTER 29 /* single slab, finisher-free loop, 2-rows/thread SpMV: launch
                               the CG SpMV in clusters of 8 CTAs that fold their p.Ap partials
                               into one through distributed shared memory (cluster-rank order),
                               so a slab of up to 8 x 4096 x 512 rows leaves <= 4096 partials and
                               the update blocks sum them without the p.Ap finisher kernel.
                               A different (fixed) summation tree: results are deterministic
                               and within the oracle tolerance, not bitwise the unclustered
                               loop's.  0 (default) off, 1 on, -1 auto (on when the unclustered
                               SpMV would leave more than 4096 partials) */
#define HPCCG_OPT_SPMV_SLICED 28 /* single slab, finisher-free loop: the CG SpMV reads a
                               CHUNK-SLICED copy of the matrix (128 rows' val[27][128] +
                               col[27][128] contiguous, built from the slot-major ELL at
                               generate time; 324 B per row of extra HBM) with ONE TMA bulk copy
                               per chunk into a two-stage shared-memory ring per persistent CTA
                               (spmv_sliced_kernel); same Ap bits; one p.Ap partial per CTA, so
                               no p.Ap finisher kernel.  0 (default) off; 1 on (allocates and
                               fills the copy); -1 auto (on when the CG vectors exceed L2).
                               Measured on two boxes: 256^3 971 / 977 vs 985 / 979
                               us/iteration, 512^3 7880 / 8048 vs 8014 / 7968 -- a gain on one
                               box, noise or a loss on the other, so not the default */
#define HPCCG_OPT_PS_LEAD 25 /* its production lead in chunks (0 default: plane/512 + 8) */
#define HPCCG_OPT_PEER_TIMEOUT_MS 22 /* HALO_PEER waits: give up after this many milliseconds
                               (1 .. 3600000; default 30000 -- above any host-side skew
                               between ranks such as graph instantiation or a slow rank) */
#define HPCCG_OPT_WHILE_UNROLL 15 /* CG iterations per execution of the WHILE body
                               (default 4: amortises the conditional node's ~8 us) */
#define HPCCG_OPT_CLUSTER_ROWS 12 /* up to this many rows (default 16384) the persistent solve
                               is ONE thread-block cluster (<= 16 CTAs) synchronised by the
                               hardware cluster barrier; above, a cooperative grid with a
                               global-memory barrier */
#define HPCCG_OPT_PDL 11    /* 1 (default): single GPU, launch the CG kernels with
                               programmatic dependent launch (the SpMV starts its matrix
                               stream while the p update drains; the SpMV lets the x/r update
                               be scheduled right after its own dependency wait, so the update
                               prefetches x, r, p during the SpMV's tail); 2: PDL with the
                               SpMV triggering only after its rows; 0: off */
#define HPCCG_OPT_SERPENTINE 20 /* single GPU, finisher-free HPCCG loop: bit 0 = the p update
                               walks the rows backwards (it starts where the x/r update ended,
                               with r and p still in L2), bit 1 = the SpMV's blocks take the row
                               blocks in reverse order.  Same rows per thread / block and the
                               same partial slots: never changes results.  -1 (default):
                               auto, 3 when the CG vectors exceed L2 (256^3), else 0 */
#define HPCCG_OPT_VEC_WAVES 6 /* CG vector kernels: 0 one thread per 16-B unit; k > 0
                               (default 1): a persistent grid of k resident waves */
#define HPCCG_OPT_SPMV_FORMAT 21 /* how the 2-rows/thread SpMV reads A: 0 (default) ELL-27,
                               val[27][n] + col[27][n] (12 B per slot); 1 DIA-27, val only:
                               slot s's column is formed from its stencil offset
                               (s/9-1)*nx*ny + (s/3%3-1)*nx + (s%3-1), a 0.0 value selecting
                               the padding column -- bitwise identical SpMV results (8 B per
                               slot).  hpccg_solve's bits are format-invariant only where both
                               formats take the same solve path: between ~9.9k and ~14k rows
                               format 1 fits the on-chip cluster solve and format 0 takes the
                               while-graph, whose reduction order differs (last bits of niters /
                               normr / x; both within the oracle tolerances).  Format 1 is an
                               "effective" reading (a different method per SURVEY 8(d)), opt-in.  Valid because hpccg_generate is the only source of
                               A (A: diag 27, -1 per existing neighbour, BJ:north_star).
                               The on-chip (shared-memory) solve drops its column slice
                               under 1 when the ELL slice does not fit (more rows on chip);
                               the 1-row/thread SpMV and the grid / one-cluster persistent
                               solves read col[]. */

typedef struct hpccg_ctx hpccg_ctx;         /* device, streams, comm (rank, nranks) */
typedef struct hpccg_problem hpccg_problem; /* A (ELL-27), b, x, x_exact, CG work vectors */

/* Per-solve statistics (filled by hpccg_solve, read with hpccg_get_stats). Times are
 * milliseconds of device time measured with CUDA events on the stream each phase
 * runs on; they are filled only with HPCCG_OPT_TIMING = 1 (else 0). */
typedef struct hpccg_stats {
    double total_ms;        /* whole solve (events around it; always filled) */
    double spmv_ms;         /* sum over SpMV launches (incl. the fused p.Ap) */
    double update_ms;       /* sum over fused x/r update + r.r launches */
    double pupdate_ms;      /* sum over p = r + beta p launches */
    double allreduce_ms;    /* sum over scalar allreduces (0 at nranks = 1) */
    double exchange_ms;     /* sum over halo exchanges (0 at nranks = 1) */
    int64_t spmv_launches;  /* SpMV passes (= niters + 1) */
    int64_t iterations;     /* niters */
    int64_t kernel_launches;/* kernels this library enqueued during the solve */
    int64_t l2_persist_bytes; /* L2 set aside for the CG vectors during the solve (0: none) */
    int64_t graph_mode;     /* 5 shared-memory-resident cluster kernel, 4 one-cluster
                               persistent kernel, 3 cooperative-grid persistent kernel,
                               2 while-graph, 1 per-iteration graph, 0 plain */
    int64_t x_deferred;     /* the deferral depth the solve ran with (HPCCG_OPT_DEFER_X): 0 none,
                               1 by one iteration, m >= 2 over a ring of m + 1 p buffers */
    int64_t ps_fused;       /* 1: the solve ran the fused p update + SpMV (HPCCG_OPT_FUSE_PSPMV) */
} hpccg_stats;

HPCCG_API const char *hpccg_strerror(int code);
HPCCG_API const char *hpccg_last_error(void);
HPCCG_API const char *hpccg_version(void);

/* Number of kernels this library has enqueued on `ctx` since hpccg_init
 * (graph replays count every kernel node).  Used for bench gpu_launches. */
HPCCG_API int hpccg_launch_count(const hpccg_ctx *ctx, int64_t *count);

/* ---------------------------------------------------------------- context */

/* Fill `out` (HPCCG_UNIQUE_ID_BYTES bytes, host) with an NCCL unique id.
 * Call on rank 0 only, then broadcast the bytes (e.g. torch.distributed).
 * HPCCG_ENOTSUP if the library was built without NCCL. */
HPCCG_API int hpccg_unique_id(void *out);

/* Create a context on CUDA `device`.  `cuda_stream` (cudaStream_t, nullable)
 * is the stream all work is enqueued on; NULL = a library-created stream.
 * unique_id == NULL: single GPU (nranks must be 1).  Otherwise z-slab rank
 * `rank` of `nranks` over NCCL; `unique_id` = the bytes from hpccg_unique_id
 * on rank 0 (north_star "z-slab decomposition ... NCCL").  nranks == 1 with a
 * unique_id runs the multi-GPU code path on a 1-rank communicator (testing).
 * Collective. */
HPCCG_API int hpccg_init(hpccg_ctx **ctx, int device, void *cuda_stream, int rank,
               int nranks, const void *unique_id);

/* Create a loopback context: all `nranks` z-slabs in this process on `device`;
 * halo exchange = device-to-device plane copies, allreduce = fixed-rank-order
 * sum kernel.  Same kernels and decomposition as the NCCL path. */
HPCCG_API int hpccg_init_loopback(hpccg_ctx **ctx, int device, void *cuda_stream,
                        int nranks);

/* Create a PEER-ONLY context: z-slab rank `rank` of `nranks`, one slab per
 * process, NO NCCL.  The CG solve's halo exchange and scalar allreduces run
 * as this library's kernels over peer memory (HPCCG_OPT_HALO_PEER) once the
 * problem is attached to its peers: every rank calls hpccg_peer_export, the
 * caller all-gathers the blobs (any transport, e.g. torch.distributed), and
 * every rank calls hpccg_peer_attach with them.  Ranks may share one GPU
 * (CUDA IPC within a device) or sit on NVLink peers.  Problem sizes are
 * global by closed form (no collective): nnz_global = (3nx-2)(3ny-2)(3 nz
 * nranks - 2).  hpccg_spmv / hpccg_ddot on caller-owned vectors need a
 * transport and return HPCCG_ENOTSUP; hpccg_maxabsdiff works after attach. */
HPCCG_API int hpccg_init_peer(hpccg_ctx **ctx, int device, void *cuda_stream, int rank, int nranks);

#define HPCCG_PEER_BLOB_BYTES 256

/* This rank's peer blob (HPCCG_PEER_BLOB_BYTES, host): CUDA IPC handles of its
 * CG vector arena and its peer-sync block.  One slab per process (NCCL or
 * peer-only contexts); not collective. */
HPCCG_API int hpccg_peer_export(hpccg_problem *prob, void *blob);

/* Map the peers' buffers from `blobs` (nranks x HPCCG_PEER_BLOB_BYTES, rank
 * order, as exported) and switch HPCCG_OPT_HALO_PEER on.  Collective over the
 * ranks in the sense that every rank must attach before any solves.  Once per
 * problem; HPCCG_EINVAL if already attached. */
HPCCG_API int hpccg_peer_attach(hpccg_problem *prob, const void *blobs);

/* rank / nranks of the context; nslabs = slabs hosted by this process
 * (1, or nranks for loopback).  NCCL contexts answer from the communicator
 * itself (ncclCommUserRank / ncclCommCount), so a bench line can show how many
 * ranks NCCL actually joined. */
HPCCG_API int hpccg_ctx_info(const hpccg_ctx *ctx, int *rank, int *nranks, int *nslabs);

HPCCG_API void hpccg_finalize(hpccg_ctx *ctx);

/* ---------------------------------------------------------------- problem */

/* a.1 -- generate this rank's slab of the HPCCG problem ON THE DEVICE
 * (HPCCG generate_matrix; north_star "on-device problem generation").
 * Global grid nx x ny x (nz * nranks); rank r owns z-planes [r nz, (r+1) nz),
 * i.e. global rows [r n, (r+1) n), n = nx ny nz, row id = z*ny*nx + y*nx + x.
 * Row i holds, for sz, sy, sx in {-1,0,1} (that nesting = ascending column),
 * the entry -1.0 (27.0 on the diagonal) iff the neighbour lies in the global
 * grid (truncated stencil, A6); b_i = 28 - nnz_i (so A.1 = b, x_exact = 1),
 * x = 0 (A5).  Storage: ELL-27 slot-major.
 * Errors: HPCCG_EINVAL if nx, ny or nz < 1 or the local row count or the
 * local-with-halo column count exceeds 2^31 - 1; HPCCG_ENOMEM. Collective. */
HPCCG_API int hpccg_generate(hpccg_ctx *ctx, int nx, int ny, int nz, hpccg_problem **out);

/* Sizes: nrow_local = n; ncol_local = n + 2 nx ny (the local-with-halo x
 * length: [lower halo plane | n owned | upper halo plane]); nnz_local = stored
 * entries of the slab(s) this process hosts; nrow_global / nnz_global over all
 * ranks.  Any out-pointer may be NULL. */
HPCCG_API int hpccg_info(const hpccg_problem *prob, int64_t *nrow_local,
               int64_t *ncol_local, int64_t *nnz_local, int64_t *nrow_global,
               int64_t *nnz_global);

/* Borrowed device pointer to X, B or XEXACT (nrow_local doubles per slab,
 * slabs concatenated in loopback mode).  Valid until hpccg_free. */
HPCCG_API int hpccg_vec(hpccg_problem *prob, int which, double **dev_ptr);

/* Copy a problem vector from / to HOST memory (nrow_local doubles per slab).
 * Pinned host memory gives full PCIe bandwidth; pageable works. */
HPCCG_API int hpccg_set_vec(hpccg_problem *prob, int which, const double *host_src);
HPCCG_API int hpccg_get_vec(const hpccg_problem *prob, int which, double *host_dst);

/* Copy slab `slab`'s ELL-27 matrix to HOST memory: val_host[27 * nrow_local]
 * and col_host[27 * nrow_local], slot-major (entry (s, i) at s*nrow_local+i),
 * columns as local-with-halo indices (global - (rank n - nx ny)); padding
 * slots hold val 0.0, col = the row's own local-with-halo index.  For tests. */
HPCCG_API int hpccg_copy_matrix(const hpccg_problem *prob, int slab, double *val_host,
                      int32_t *col_host);

HPCCG_API int hpccg_set_option(hpccg_problem *prob, int key, int64_t value);

/* ------------------------------------------------------------- operations */

/* a.2 + a.3 -- y = A x (HPCCG HPC_sparsemv; the paper's analogue is the
 * matvecmul of Fig. 12).  x: device, ncol_local doubles in the
 * local-with-halo layout; its two halo planes are OVERWRITTEN by the halo
 * exchange this call performs (zero-filled at the global z boundary).
 * y: device, nrow_local doubles; must not overlap x.  Per row, the stored
 * entries are reduced in ascending column order as an fp64 FMA chain from
 * +0.0 (A8), so the result is bitwise reproducible. */
HPCCG_API int hpccg_spmv(hpccg_problem *prob, double *x, double *y);

/* a.4/a.10 -- *result (HOST) = sum_i x_i y_i over all ranks (JACC DOT: Fig. 2
 * P:L67-L69; HPCCG ddot + MPI_Allreduce).  x, y: device, n doubles
 * each (x == y allowed).  Local sum: deterministic fixed-shape tree; then a
 * sum-allreduce in fixed rank order (loopback) or via NCCL.  n >= 0. */
HPCCG_API int hpccg_ddot(hpccg_ctx *ctx, int64_t n, const double *x, const double *y,
               double *result);

/* a.5/a.6/a.10 -- w = alpha x + beta y (HPCCG waxpby; JACC AXPY x += alpha y
 * of Fig. 2 P:L64-L66 is hpccg_waxpby(n, 1, x, alpha, y, x)).  Device arrays
 * of n doubles; w may alias x or y.  Canonical single-FMA forms (A10):
 * alpha == 1 -> fma(beta, y, x); beta == 1 -> fma(alpha, x, y); otherwise
 * fma(alpha, x, beta * y).  Purely local (no communication). */
HPCCG_API int hpccg_waxpby(hpccg_ctx *ctx, int64_t n, double alpha, const double *x,
                 double beta, const double *y, double *w);

/* f3 -- JACC's multidimensional constructs on 2-D arrays (Fig. 2):
 * column-major m x n arrays with leading dimension ld >= m (element (i, j) at
 * i + j*ld; only the m x n block is touched).  waxpby2d: w = alpha x + beta y
 * with the canonical forms of hpccg_waxpby (JACC's 2-D axpy x[i,j] += alpha
 * y[i,j] is waxpby2d(m, n, ld, 1, x, alpha, y, x)); ddot2d: *result (HOST) =
 * sum over (i, j) of x[i,j] y[i,j] over all ranks (deterministic tree +
 * allreduce).  Loopback: the per-rank arrays are stacked (ld*n doubles each). */
HPCCG_API int hpccg_waxpby2d(hpccg_ctx *ctx, int64_t m, int64_t n, int64_t ld, double alpha,
                             const double *x, double beta, const double *y, double *w);
HPCCG_API int hpccg_ddot2d(hpccg_ctx *ctx, int64_t m, int64_t n, int64_t ld, const double *x,
                           const double *y, double *result);

/* a.2-a.8 -- HPCCG's unpreconditioned CG (the paper's loop Fig. 12
 * P:L450-L474; loop semantics A3/A4):
 *   p = x; Ap = A p; r = b - Ap; rtrans = r.r; normr = sqrt(rtrans)
 *   for (k = 1; k < max_iter && normr > tol; k++):
 *     k == 1 ? p = r : { beta = (r.r) / rtrans_old; p = r + beta p }
 *     normr = sqrt(rtrans); Ap = A p; alpha = rtrans / p.Ap;
 *     x += alpha p; r -= alpha Ap; niters = k
 * with guard A11 (rtrans == 0 or p.Ap == 0 -> alpha = 0, stop).  Uses the
 * problem's b; the problem's X is the initial guess in and the iterate out.
 * All scalars (alpha, beta, normr, stop flag) live on the device; no per-dot
 * host round trip.  *niters, *normr: HOST out (nullable).  times (HOST,
 * nullable, 6 entries, seconds): total, ddot, waxpby, spmv, allreduce,
 * exchange -- phase entries need HPCCG_OPT_TIMING = 1 (ddot is fused into the
 * waxpby/spmv kernels, so times[1] = 0).  max_iter >= 1, tol >= 0. */
HPCCG_API int hpccg_solve(hpccg_problem *prob, int max_iter, double tol, int *niters,
                double *normr, double times[6]);

/* Device trace of the last solve (HPCCG_OPT_TRACE = k): out[(i*3 + j)*2 + {0,1}]
 * = start / end (ns, device clock) of kernel j (0 p update, 1 SpMV, 2 x/r update)
 * in iteration i+1, for i < min(k, niters); 0 where a kernel did not run.
 * `out` (HOST) holds 6*k uint64.  Single slab / first slab. */
HPCCG_API int hpccg_get_trace(const hpccg_problem *prob, uint64_t *out, int64_t k);

/* Statistics of the last hpccg_solve on `prob`. */
HPCCG_API int hpccg_get_stats(const hpccg_problem *prob, hpccg_stats *out);

/* a.9 -- *result (HOST) = max_i |x_i - x_exact_i| over all ranks (HPCCG
 * compute_residual; north_star "final max|x-1|"). */
HPCCG_API int hpccg_maxabsdiff(hpccg_problem *prob, double *result);

HPCCG_API void hpccg_free(hpccg_problem *prob);

/* ---------------------------------------------------------------------------
 * f1 -- the paper's own CG workload: Fig. 12, an
 * unpreconditioned CG on a "diagonal-dominant tridiagonal" matrix
 * held as three coefficient arrays a0 (sub), a1 (diag), a2 (super), read as
 * tridiag(1, 4, 1) (A18); initial state r = p = b = 0.5 * 1, x = 0
 * (P:L475-L484); the loop runs while cond = r.r > tol (A3) and at most
 * max_iter times.  The paper times one iteration at SIZE = 1e8.
 * Single GPU only (the paper's runs are single-device): ENOTSUP on a
 * multi-rank or loopback context.
 * ------------------------------------------------------------------------- */
typedef struct hpccg_tri hpccg_tri;

#define HPCCG_TRI_X 0
#define HPCCG_TRI_B 1
#define HPCCG_TRI_R 2
#define HPCCG_TRI_P 3
#define HPCCG_TRI_A0 4
#define HPCCG_TRI_A1 5
#define HPCCG_TRI_A2 6

/* Generate the size-n system on the device (a0[0] = a2[n-1] = 0).  Caller
 * frees with hpccg_tri_free.  EINVAL if n < 1. */
HPCCG_API int hpccg_tri_generate(hpccg_ctx *ctx, int64_t n, hpccg_tri **out);

/* Borrowed device pointer (n doubles) to X, B, R, P or a coefficient array
 * (P: the buffer holding the last solve's final p -- a ring slot after a
 * variant-2 solve). */
HPCCG_API int hpccg_tri_vec(hpccg_tri *t, int which, double **dev_ptr);

/* y = A x (Fig. 12 matvecmul): y_i = a0_i x_{i-1} + a1_i x_i + a2_i x_{i+1}
 * over the existing terms, ascending column, fp64 FMA chain from +0.0 (A8).
 * x, y: device, n doubles, not overlapping. */
HPCCG_API int hpccg_tri_spmv(hpccg_tri *t, const double *x, double *y);

/* Reset x = 0, r = p = b and run the CG.  variant 0: the iteration exactly as
 * Fig. 12 writes it -- copy r_old, matvec, 5 dots, 3 axpys (axpy(i, a, x, y):
 * x[i] += a*y[i]), 2 more copies -- with every scalar on the device; variant
 * 1: fused (matvec + p.s, x/r update + r.r, p update: 112n B per iteration);
 * variant 2: variant 1 with x += alpha_k p_k deferred over 8 iterations
 * through a ring of 9 p buffers (p_k in slot (k - 1) % 9; x read and written
 * once per 8 iterations, the pending directions applied after the loop: 97n
 * B per iteration, 8 more p-sized device buffers allocated on first use) --
 * the same FMAs on x in the same order, so bitwise variant 1's x, iterations,
 * r.r and p.  All run as one graph with a device-driven WHILE node.  *iters,
 * *cond (last r.r), *ms (device time of the whole solve): HOST out, nullable.
 * EINVAL for another variant. */
HPCCG_API int hpccg_tri_solve(hpccg_tri *t, int max_iter, double tol, int variant, int *iters,
                              double *cond, double *ms);

HPCCG_API void hpccg_tri_free(hpccg_tri *t);

/* ---------------------------------------------------------------------------
 * f4 -- the paper's third workload: the 2-lattice D2Q9 "pull"
 * lattice-Boltzmann step of Fig. 10 / Eq. (1) on an
 * S x S lattice (S = 1000 in the paper).  State: 9 S^2 doubles,
 * distribution k of site (x, y) at k*S*S + x*S + y (y fastest); lattice
 * c_k, w_k and the equilibrium as read in DESIGN.md A21-A24.  Lattice 0 is
 * the current state, 1 the next, 2 the streamed f of the last step (written
 * only when write_f).  Only interior sites 1 <= x, y <= S-2 are updated.
 * Single GPU only (ENOTSUP otherwise).
 * ------------------------------------------------------------------------- */
typedef struct hpccg_lbm hpccg_lbm;

/* Allocate the three zero-filled lattices (S >= 3). */
HPCCG_API int hpccg_lbm_create(hpccg_ctx *ctx, int size, hpccg_lbm **out);
/* Copy lattice `which` (0 current, 1 next, 2 streamed f) from / to HOST memory. */
HPCCG_API int hpccg_lbm_set(hpccg_lbm *l, int which, const double *host);
HPCCG_API int hpccg_lbm_get(const hpccg_lbm *l, int which, double *host);
/* `steps` steps with relaxation time tau > 0: each step pulls lattice 0 into
 * lattice 1 (Fig. 10's f1 -> f2), then the two trade places, so lattice 0 is
 * always the newest state.  *ms (HOST, nullable) = device time.
 * write_f: bit 0 materialises the streamed f into lattice 2; the other bits
 * are tuning knobs (bits 1-2 cache policy, bit 3 no PDL; bit 4 runs the steps
 * in fused pairs -- two steps per kernel, the intermediate lattice on chip,
 * same bits; lattice 1 then keeps only its boundary sites and lattice 2 is
 * scratch; ignored with bit 0). */
HPCCG_API int hpccg_lbm_run(hpccg_lbm *l, int steps, double tau, int write_f, double *ms);
HPCCG_API void hpccg_lbm_free(hpccg_lbm *l);

#ifdef __cplusplus
}
#endif

#endif /* HPCCG_H */
