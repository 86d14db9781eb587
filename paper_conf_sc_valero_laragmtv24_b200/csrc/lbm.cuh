// lbm.cuh -- sm_100a kernels of the paper's third workload: the
// 2-lattice D2Q9 "pull" lattice-Boltzmann step of Fig. 10,
// Eq. (1).  Per interior site: 9 pulled loads of f1, moments, BGK
// relaxation, 9 stores of f2 (+9 of the streamed f when it is materialised)
// -> 144 B/site (216).
// The arithmetic is written with explicit round-to-nearest intrinsics in the
// order of the oracle (A21-A24), so no FMA contraction can change
// a bit: GPU and oracle agree bitwise.  The only rewrites are exact ones:
// c*a for a lattice constant c = +-1 is +-a, and operations that repeat with
// identical operands (w_k p for equal weights, the opposite direction's
// (4.5 cu) cu and 3 cu, whose signs flip exactly) are computed once.
// Included by hpccg.cu.
#pragma once

#include "kernels.cuh"

namespace hpccg {

// D2Q9 lattice (A22): c = (0,0), (1,0), (0,1), (-1,0), (0,-1), (1,1), (-1,1), (-1,-1), (1,-1)
__host__ __device__ constexpr int lbm_cx(int k) { return (k == 1 || k == 5 || k == 8) ? 1 : (k == 3 || k == 6 || k == 7) ? -1 : 0; }
__host__ __device__ constexpr int lbm_cy(int k) { return (k == 2 || k == 5 || k == 6) ? 1 : (k == 4 || k == 7 || k == 8) ? -1 : 0; }

// RN(a * c) for c in {-1, 0, 1}: exact sign copies for +-1, a real multiply for 0
// (0 * a is -0, +0 or NaN depending on a -- kept as the oracle computes it)
__device__ __forceinline__ double lbm_cmul(double a, int c) {
    return c == 1 ? a : (c == -1 ? -a : __dmul_rn(a, 0.0));
}

// One site of Fig. 10 from its 9 pulled values fk: out_k = fk (1 - 1/t) + feq_k / t,
// keep = 1 - 1/t (computed once on the host, same IEEE operations).  Operation
// order = oracle_lbm_step / oracle_lbm_feq.
__device__ __forceinline__ void lbm_collide(const double (&fk)[9], double keep, double tau,
                                            double (&out)[9]) {
    double p = 0.0, u = 0.0, v = 0.0;
#pragma unroll
    for (int k = 0; k < 9; ++k) {
        p = __dadd_rn(p, fk[k]);
        u = __dadd_rn(u, lbm_cmul(fk[k], lbm_cx(k)));
        v = __dadd_rn(v, lbm_cmul(fk[k], lbm_cy(k)));
    }
    u = __ddiv_rn(u, p);
    v = __ddiv_rn(v, p);
    const double usq = __dadd_rn(__dmul_rn(u, u), __dmul_rn(v, v));
    const double h = __dmul_rn(1.5, usq);
    // w_k p for the three weights (4/9, 1/9, 1/36)
    const double wp0 = __dmul_rn(4.0 / 9, p), wp1 = __dmul_rn(1.0 / 9, p), wp5 = __dmul_rn(1.0 / 36, p);
    // cu, 3 cu and (4.5 cu) cu for k = 0, 1, 2, 5, 6; k = 3, 4, 7, 8 are the opposites of
    // 1, 2, 5, 6: cu flips sign exactly, so does 3 cu, and (4.5 cu) cu is unchanged
    double cu[9], t3[9], q[9];
#pragma unroll
    for (int k = 0; k < 9; ++k) {
        if (k == 3 || k == 4 || k == 7 || k == 8) continue;
        cu[k] = __dadd_rn(lbm_cmul(u, lbm_cx(k)), lbm_cmul(v, lbm_cy(k)));
        t3[k] = __dmul_rn(3.0, cu[k]);
        q[k] = __dmul_rn(__dmul_rn(4.5, cu[k]), cu[k]);
    }
    t3[3] = -t3[1]; q[3] = q[1];
    t3[4] = -t3[2]; q[4] = q[2];
    t3[7] = -t3[5]; q[7] = q[5];
    t3[8] = -t3[6]; q[8] = q[6];
#pragma unroll
    for (int k = 0; k < 9; ++k) {
        double t = __dadd_rn(1.0, t3[k]);
        t = __dadd_rn(t, q[k]);
        t = __dsub_rn(t, h);
        const double wp = k == 0 ? wp0 : (k < 5 ? wp1 : wp5);
        const double feq = __dmul_rn(wp, t);
        out[k] = __dadd_rn(__dmul_rn(fk[k], keep), __ddiv_rn(feq, tau));
    }
}

// kPol: cache policy of the lattice streams -- 0: loads and stores
// streaming (evict-first); 1 (default): loads streaming, stores cached (the
// lattice just written, 72 MB at 1000^2, stays largely in the 126 MB L2 for
// the next step's pulls: 26.7 vs 29.3 us/step measured); 2: both cached.
#ifndef HPCCG_LBM_MINB
#define HPCCG_LBM_MINB 4  // 64 registers, 4 CTAs/SM: 21.45 vs 25.13 us/step at 1000^2 (68 regs, 3 CTAs); 5-6 spill
#endif
template <bool kWriteF, int kPol>
__global__ void __launch_bounds__(kBlock, HPCCG_LBM_MINB) lbm_pull_kernel(int S, const double *__restrict__ f1,
                                                         double *__restrict__ f,
                                                         double *__restrict__ f2, double keep,
                                                         double tau) {
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
    double fk[9], out[9];
#pragma unroll
    for (int k = 0; k < 9; ++k) {
        const int xs = x - lbm_cx(k), ys = y - lbm_cy(k);
        const double *src = f1 + k * SS + (int64_t)xs * S + ys;
        fk[k] = kPol == 2 ? __ldg(src) : __ldcs(src);
    }
    if (kWriteF) {
#pragma unroll
        for (int k = 0; k < 9; ++k) __stcs(f + k * SS + site, fk[k]);
    }
    lbm_collide(fk, keep, tau, out);
#pragma unroll
    for (int k = 0; k < 9; ++k) {
        if (kPol == 0) __stcs(f2 + k * SS + site, out[k]);
        else f2[k * SS + site] = out[k];
    }
}

// ---------------------------------------------------------------------------
// Two steps per kernel (temporal blocking; opt-in tuning bit 4, `write_f` = 0
// only -- measured slower than two single steps at 1000^2: 25.7 vs 25.0
// us/step at best, the doubled per-CTA FP64 work (2 x 216 DP operations per
// site, 12 of them divisions) runs at 16 warps/SM and is not hidden).  Step 1 pulls
// lattice A into an on-chip ring of rows, step 2 pulls that ring into lattice
// C: one HBM read of A and one write of C per two steps (72 B/site/step
// instead of 144).  A CTA owns a strip of kLbmCols output columns and a chunk
// of `rows` output rows; it marches down the chunk computing step-1 row r
// (kLbmCols + 2 columns: its own and one halo column each side) and then
// step-2 row r - 1 from ring rows r - 2 .. r.  Step-1 values of boundary
// sites are lattice B's boundary values (Fig. 10 never updates them); halo
// rows / columns are recomputed by the neighbouring CTAs (extra work
// (rows + 2) / rows x 128 / 126).  Results are the two sequential steps'
// bits exactly (same per-site operations).  The intermediate lattice never
// reaches HBM, so lattice B's interior is not updated.
constexpr int kLbmT = 128;             // threads per CTA = step-1 columns
constexpr int kLbmCols = kLbmT - 2;    // output columns per CTA

template <int kMinB>
__global__ void __launch_bounds__(kLbmT, kMinB) lbm_pull2_kernel(int S, int rows,
                                                         const double *__restrict__ A,
                                                         const double *__restrict__ B,
                                                         double *__restrict__ C, double keep,
                                                         double tau) {
    __shared__ double ring[4][9][kLbmT];
    const int64_t SS = (int64_t)S * S;
    const int t = threadIdx.x;
    const int c = (int)blockIdx.x * kLbmCols + t;          // column (ys - 1 + t, ys = 1 + strip * 126)
    const int xa = 1 + (int)blockIdx.y * rows;
    const int xb = min(xa + rows, S - 1);                  // output rows [xa, xb)
    const bool col_in = c >= 1 && c <= S - 2;
    const bool col_ok = c <= S - 1;
    const bool out_col = col_in && t >= 1 && t <= kLbmCols;
    pdl_wait();
    pdl_trigger();
    // step-1 inputs of row r: the 9 pulls of A (interior), B's value (boundary), 0 (outside)
    auto load_row = [&](int r, double (&v)[9]) {
        if (col_in && r >= 1 && r <= S - 2) {
#pragma unroll
            for (int k = 0; k < 9; ++k)
                v[k] = __ldcs(A + k * SS + (int64_t)(r - lbm_cx(k)) * S + (c - lbm_cy(k)));
        } else if (col_ok && r >= 0 && r <= S - 1) {
#pragma unroll
            for (int k = 0; k < 9; ++k) v[k] = __ldg(B + k * SS + (int64_t)r * S + c);
        } else {
#pragma unroll
            for (int k = 0; k < 9; ++k) v[k] = 0.0;
        }
    };
    double cur[9];
    load_row(xa - 1, cur);
    for (int r = xa - 1; r <= xb; ++r) {
        double nxt[9];
        if (r < xb) load_row(r + 1, nxt);  // prefetch the next row during this row's math
        double s1[9];
        if (col_in && r >= 1 && r <= S - 2) {
            lbm_collide(cur, keep, tau, s1);
        } else {
#pragma unroll
            for (int k = 0; k < 9; ++k) s1[k] = cur[k];
        }
#pragma unroll
        for (int k = 0; k < 9; ++k) ring[r & 3][k][t] = s1[k];
        __syncthreads();
        const int x = r - 1;  // step-2 row: ring rows x - 1, x, x + 1 = r - 2 .. r
        if (x >= xa && out_col) {
            double fk[9], o[9];
#pragma unroll
            for (int k = 0; k < 9; ++k) fk[k] = ring[(x - lbm_cx(k)) & 3][k][t - lbm_cy(k)];
            lbm_collide(fk, keep, tau, o);
#pragma unroll
            for (int k = 0; k < 9; ++k) C[k * SS + (int64_t)x * S + c] = o[k];
        }
        if (r < xb) {
#pragma unroll
            for (int k = 0; k < 9; ++k) cur[k] = nxt[k];
        }
    }
}

// dst's boundary sites (x or y in {0, S-1}) := src's, all 9 distributions
__global__ void __launch_bounds__(kBlock) lbm_edge_copy_kernel(int S, const double *__restrict__ src,
                                                              double *__restrict__ dst) {
    pdl_wait();
    pdl_trigger();
    const int64_t SS = (int64_t)S * S;
    const int64_t per = 4 * (int64_t)S;  // rows 0 and S-1 (S each), columns 0 and S-1 (S each)
    for (int64_t i = gtid(); i < 9 * per; i += gnth()) {
        const int k = (int)(i / per);
        const int64_t j = i - k * per;
        const int side = (int)(j / S), m = (int)(j - (int64_t)side * S);
        const int x = side == 0 ? 0 : side == 1 ? S - 1 : m;
        const int y = side < 2 ? m : (side == 2 ? 0 : S - 1);
        const int64_t o = k * SS + (int64_t)x * S + y;
        dst[o] = src[o];
    }
}

}  // namespace hpccg
