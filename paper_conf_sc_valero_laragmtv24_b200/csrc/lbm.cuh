// lbm.cuh -- sm_100a kernel of the paper's third workload: the
// 2-lattice D2Q9 "pull" lattice-Boltzmann step of Fig. 10,
// Eq. (1).  One thread per lattice site (y fastest, coalesced);
// per interior site: 9 pulled loads of f1, moments, BGK relaxation, 9 stores
// of f2 (+9 of the streamed f when it is materialised) -> 144 B/site (216).
// The arithmetic is written with explicit round-to-nearest intrinsics in the
// order of the oracle (A21-A24), so no FMA contraction can change
// a bit: GPU and oracle agree bitwise.  Included by hpccg.cu.
#pragma once

#include "kernels.cuh"

namespace hpccg {

__constant__ double kLbmCx[9] = {0, 1, 0, -1, 0, 1, -1, -1, 1};
__constant__ double kLbmCy[9] = {0, 0, 1, 0, -1, 1, 1, -1, -1};
__constant__ double kLbmW[9] = {4.0 / 9, 1.0 / 9, 1.0 / 9, 1.0 / 9, 1.0 / 9,
                                1.0 / 36, 1.0 / 36, 1.0 / 36, 1.0 / 36};

// kPol: cache policy of the lattice streams -- 0: loads and stores
// streaming (evict-first); 1 (default): loads streaming, stores cached (the
// lattice just written, 72 MB at 1000^2, stays largely in the 126 MB L2 for
// the next step's pulls: 26.7 vs 29.3 us/step measured); 2: both cached.
template <bool kWriteF, int kPol>
__global__ void __launch_bounds__(kBlock) lbm_pull_kernel(int S, const double *__restrict__ f1,
                                                         double *__restrict__ f,
                                                         double *__restrict__ f2, double tau) {
    // grid (ceil((S-2)/256), S-2): blockIdx.y -> row x, threads -> y (interior only, Fig. 10)
    const int64_t SS = (int64_t)S * S;
    const int x = 1 + (int)blockIdx.y;
    const int y = 1 + (int)(blockIdx.x * kBlock + threadIdx.x);
    // PDL: this step's blocks are scheduled during the previous step's tail
    // and wait here until it has completed (every pull may read its output)
    pdl_wait();
    pdl_trigger();
    if (y > S - 2) return;
    const int64_t site = (int64_t)x * S + y;
    double fk[9];
#pragma unroll
    for (int k = 0; k < 9; ++k) {
        const int xs = x - (int)kLbmCx[k], ys = y - (int)kLbmCy[k];
        const double *src = f1 + k * SS + (int64_t)xs * S + ys;
        fk[k] = kPol == 2 ? __ldg(src) : __ldcs(src);
    }
    if (kWriteF) {
#pragma unroll
        for (int k = 0; k < 9; ++k) __stcs(f + k * SS + site, fk[k]);
    }
    double p = 0.0, u = 0.0, v = 0.0;
#pragma unroll
    for (int k = 0; k < 9; ++k) {
        p = __dadd_rn(p, fk[k]);
        u = __dadd_rn(u, __dmul_rn(fk[k], kLbmCx[k]));
        v = __dadd_rn(v, __dmul_rn(fk[k], kLbmCy[k]));
    }
    u = __ddiv_rn(u, p);
    v = __ddiv_rn(v, p);
    const double usq = __dadd_rn(__dmul_rn(u, u), __dmul_rn(v, v));
    const double keep = __dsub_rn(1.0, __ddiv_rn(1.0, tau));  // (1 - 1/t)
#pragma unroll
    for (int k = 0; k < 9; ++k) {
        const double cu = __dadd_rn(__dmul_rn(kLbmCx[k], u), __dmul_rn(kLbmCy[k], v));
        double t = __dadd_rn(1.0, __dmul_rn(3.0, cu));
        t = __dadd_rn(t, __dmul_rn(__dmul_rn(4.5, cu), cu));
        t = __dsub_rn(t, __dmul_rn(1.5, usq));
        const double feq = __dmul_rn(__dmul_rn(kLbmW[k], p), t);
        const double out = __dadd_rn(__dmul_rn(fk[k], keep), __ddiv_rn(feq, tau));
        if (kPol == 0) __stcs(f2 + k * SS + site, out);
        else f2[k * SS + site] = out;
    }
}

}  // namespace hpccg
