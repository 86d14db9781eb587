// tridiag.cuh -- sm_100a kernels of the paper's own CG workload:
// Fig. 12, a diagonal-dominant tridiagonal matrix held as three
// coefficient arrays (read as tridiag(1, 4, 1), A18), SIZE = 1e8,
// one CG iteration timed.  Two iteration structures:
//   variant 0 -- Fig. 12 as written: 3 copies, 1 matvec, 5 dots, 3 axpys per
//                iteration (12 kernels + 1 control kernel), scalars on device;
//   variant 1 -- fused: matvec + p.s, x/r update + r.r, p update (3 kernels);
//   variant 2 -- variant 1 with x deferred over kTriM iterations (a ring of
//                kTriM + 1 p buffers, the same FMAs on x in the same order:
//                bitwise variant 1's results) -- 97n instead of 112n B.
// Included by hpccg.cu (one translation unit).
#pragma once

#include "kernels.cuh"

namespace hpccg {

constexpr int kTriU = 4;  // elements per thread per trip, all loads first

struct TriScalars {
    double slot[5];   // variant 0: alpha0, alpha1, beta0, beta1, cond
    double rr;        // variant 1: r.r of the current r
    double pAp;       // variant 1: p.s
    double cond;      // last r.r (both variants)
    double tol;
    int it;           // iterations done
    int max_iter;
    double alpha_h[16];  // variant 2: alpha of iteration k in slot k & 15
};

// variant 2: p_k (iteration k's direction) lives in slot (k - 1) % (m + 1);
// slot 0 is the problem's p buffer (the init writes p_1 = b there), slots
// j >= 1 at base + (j - 1) stride.  m == 0: no ring (variants 0 / 1).
constexpr int kTriM = 8;
struct TriRing {
    double *p0, *base;
    int64_t stride;
    int m;
};

__host__ __device__ __forceinline__ double *tri_slot(const TriRing &g, int j) {
    return j == 0 ? g.p0 : g.base + (int64_t)(j - 1) * g.stride;
}

// a0[i] = 1 (i > 0), a1[i] = 4, a2[i] = 1 (i < n-1), zero outside; b = 0.5.
__global__ void __launch_bounds__(kBlock) tri_gen_kernel(int64_t n, double *a0, double *a1, double *a2,
                                                        double *b) {
    for (int64_t i = gtid(); i < n; i += gnth()) {
        a0[i] = i > 0 ? 1.0 : 0.0;
        a1[i] = 4.0;
        a2[i] = i < n - 1 ? 1.0 : 0.0;
        b[i] = 0.5;
    }
}

// matvecmul (Fig. 12): y_i = a0_i x_{i-1} + a1_i x_i + a2_i x_{i+1}, existing
// terms, ascending column, FMA chain from +0.0 (A8).  kDot: partial x.y into
// the deterministic grid reduction -> *dot_out.  40n B (+0: x neighbours hit L1).
template <bool kDot>
__global__ void __launch_bounds__(kBlock) tri_spmv_kernel(int64_t n, const double *__restrict__ a0,
                                                         const double *__restrict__ a1,
                                                         const double *__restrict__ a2,
                                                         const double *__restrict__ x,
                                                         double *__restrict__ y, Reduction red,
                                                         double *dot_out, TriRing g = TriRing{},
                                                         const TriScalars *sc = nullptr) {
    const uint64_t pol = policy_evict_first();
    pdl_wait();
    pdl_trigger();
    // variant 2: iteration it + 1 gathers p_(it+1) from slot it % (m + 1)
    if (g.m >= 2) x = tri_slot(g, ldg_o(&sc->it) % (g.m + 1));
    double d = 0.0;
    const int64_t nth = gnth();
    for (int64_t b0 = gtid(); b0 < n; b0 += kTriU * nth) {
        double c0[kTriU], c1[kTriU], c2[kTriU], xm[kTriU], xi[kTriU], xp[kTriU];
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) {
                c0[u] = ld_stream(a0 + i, pol);
                c1[u] = ld_stream(a1 + i, pol);
                c2[u] = ld_stream(a2 + i, pol);
                xm[u] = i > 0 ? x[i - 1] : 0.0;
                xi[u] = x[i];
                xp[u] = i < n - 1 ? x[i + 1] : 0.0;
            }
        }
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) {
                double s = 0.0;
                if (i > 0) s = fma(c0[u], xm[u], s);
                s = fma(c1[u], xi[u], s);
                if (i < n - 1) s = fma(c2[u], xp[u], s);
                y[i] = s;
                if (kDot) d = fma(xi[u], s, d);
            }
        }
    }
    if (kDot) grid_reduce<false>(d, red, blockIdx.x, gridDim.x, [dot_out](double v) { *dot_out = v; });
}

// JACC axpy(i, alpha, x, y): x[i] += alpha * y[i] = fma(alpha, y, x) (A10), with
// alpha = sign * (*num / *den) read from device scalars ("negative_alpha =
// alpha * (-1.0)").  24n B.
__global__ void __launch_bounds__(kBlock) tri_axpy_kernel(int64_t n, double *__restrict__ x,
                                                         const double *__restrict__ y,
                                                         const double *num, const double *den,
                                                         double sign) {
    pdl_wait();
    pdl_trigger();
    const double alpha = (__ldg(num) / __ldg(den)) * sign;
    const int64_t nth = gnth();
    for (int64_t b0 = gtid(); b0 < n; b0 += kTriU * nth) {
        double xv[kTriU], yv[kTriU];
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) {
                xv[u] = x[i];
                yv[u] = y[i];
            }
        }
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) x[i] = fma(alpha, yv[u], xv[u]);
        }
    }
}

__global__ void __launch_bounds__(kBlock) tri_copy_kernel(int64_t n, const double *__restrict__ src,
                                                         double *__restrict__ dst) {
    pdl_wait();
    pdl_trigger();
    const int64_t nth = gnth();
    for (int64_t b0 = gtid(); b0 < n; b0 += kTriU * nth) {
        double v[kTriU];
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) v[u] = src[i];
        }
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) dst[i] = v[u];
        }
    }
}

// dot for variant 0 (each of Fig. 12's five parallel_reduce calls) -> *out
__global__ void __launch_bounds__(kBlock) tri_dot_kernel(int64_t n, const double *__restrict__ x,
                                                        const double *__restrict__ y, Reduction red,
                                                        double *out) {
    pdl_wait();
    pdl_trigger();
    double acc = 0.0;
    const int64_t nth = gnth();
    const int64_t full = n / (kTriU * nth) * (kTriU * nth);  // trips where all kTriU are in range
    int64_t b0 = gtid();
    for (; b0 < full; b0 += kTriU * nth) {
        double xv[kTriU], yv[kTriU];
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            xv[u] = x[b0 + u * nth];
            yv[u] = y[b0 + u * nth];
        }
#pragma unroll
        for (int u = 0; u < kTriU; ++u) acc = fma(xv[u], yv[u], acc);
    }
    // ragged tail (n - full < kTriU * nth: at most kTriU per thread), same
    // order, a fixed trip count so no lane leaves early
#pragma unroll
    for (int t = 0; t < kTriU; ++t) {
        const int64_t i = b0 + t * nth;
        if (i < n) acc = fma(x[i], y[i], acc);
    }
    grid_reduce<false>(acc, red, blockIdx.x, gridDim.x, [out](double v) { *out = v; });
}

// loop control of variant 0: cond = r.r (slot 4); it++; continue while
// cond > tol and it < max_iter (A3 reading of Fig. 12's loop).
__global__ void tri_ctrl_kernel(TriScalars *sc, unsigned long long cond_handle) {
    pdl_wait();
    const double c = sc->slot[4];
    const int it = sc->it + 1;
    sc->it = it;
    sc->cond = c;
    set_cond(cond_handle, c > sc->tol && it < sc->max_iter);
}

// init: x = 0, r = p = b (0.5), s = 0; cond = 1.0; it = 0.
__global__ void __launch_bounds__(kBlock) tri_init_kernel(int64_t n, const double *__restrict__ b,
                                                         double *x, double *r, double *p, double *s) {
    for (int64_t i = gtid(); i < n; i += gnth()) {
        x[i] = 0.0;
        r[i] = b[i];
        p[i] = b[i];
        s[i] = 0.0;
    }
}

__global__ void tri_initstate_kernel(TriScalars *sc, int max_iter, double tol, int fused,
                                     unsigned long long cond_handle) {
    sc->it = 0;
    sc->cond = 1.0;  // Fig. 12: cond = 1.0 before the loop
    sc->tol = tol;
    sc->max_iter = max_iter;
    set_cond(cond_handle, 1.0 > tol && 0 < max_iter);
    (void)fused;
}

// variant 1, init of rr = r.r (the fused loop carries it)
__global__ void __launch_bounds__(kBlock) tri_rr_kernel(int64_t n, const double *__restrict__ r,
                                                       Reduction red, TriScalars *sc) {
    double acc = 0.0;
    for (int64_t i = gtid(); i < n; i += gnth()) acc = fma(r[i], r[i], acc);
    grid_reduce<false>(acc, red, blockIdx.x, gridDim.x, [sc](double v) { sc->rr = v; });
}

// variant 1: alpha = rr / p.s; r = fma(-alpha, s, r); x = fma(alpha, p, x);
// r.r -> last block: beta = rr_new / rr, cond = rr_new, it++, loop control.
// kDefer (variant 2): x is left to the p updates (alpha -> sc->alpha_h), so
// this pass reads s, r and writes r only (24n instead of 48n B)
template <bool kDefer = false>
__global__ void __launch_bounds__(kBlock) tri_update_kernel(int64_t n, double *__restrict__ x,
                                                           double *__restrict__ r,
                                                           const double *__restrict__ p,
                                                           const double *__restrict__ s,
                                                           Reduction red, TriScalars *sc,
                                                           unsigned long long cond_handle) {
    pdl_wait();
    pdl_trigger();
    const double rr = ldg_o(&sc->rr);
    const double alpha = rr / ldg_o(&sc->pAp);
    const double nalpha = alpha * (-1.0);
    if (kDefer && blockIdx.x == 0 && threadIdx.x == 0) sc->alpha_h[(ldg_o(&sc->it) + 1) & 15] = alpha;
    double acc = 0.0;
    const int64_t nth = gnth();
    for (int64_t b0 = gtid(); b0 < n; b0 += kTriU * nth) {
        double sv[kTriU], rv[kTriU], pv[kTriU], xv[kTriU];
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) {
                sv[u] = s[i];
                rv[u] = r[i];
                if (!kDefer) {
                    pv[u] = p[i];
                    xv[u] = x[i];
                }
            }
        }
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) {
                const double rn = fma(nalpha, sv[u], rv[u]);
                r[i] = rn;
                if (!kDefer) x[i] = fma(alpha, pv[u], xv[u]);
                acc = fma(rn, rn, acc);
            }
        }
    }
    grid_reduce<false>(acc, red, blockIdx.x, gridDim.x, [sc, rr, cond_handle](double v) {
        sc->slot[2] = v / rr;  // beta = beta0 / beta1 (beta1 = r_old.r_old = rr)
        sc->rr = v;
        sc->cond = v;
        const int it = sc->it + 1;
        sc->it = it;
        set_cond(cond_handle, v > sc->tol && it < sc->max_iter);
    });
}

// variant 1: p = r + beta p (r_aux = r; r_aux += beta p; p = r_aux) = fma(beta, p, r)
__global__ void __launch_bounds__(kBlock) tri_pupdate_kernel(int64_t n, const double *__restrict__ r,
                                                            double *__restrict__ p,
                                                            const TriScalars *sc) {
    pdl_wait();
    pdl_trigger();
    const double beta = ldg_o(&sc->slot[2]);
    const int64_t nth = gnth();
    for (int64_t b0 = gtid(); b0 < n; b0 += kTriU * nth) {
        double pv[kTriU], rv[kTriU];
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) {
                pv[u] = p[i];
                rv[u] = r[i];
            }
        }
#pragma unroll
        for (int u = 0; u < kTriU; ++u) {
            const int64_t i = b0 + u * nth;
            if (i < n) p[i] = fma(beta, pv[u], rv[u]);
        }
    }
}

// variant 2: p_(k+1) = r + beta p_k into slot k % (m + 1) (k = it, after the
// update of iteration k); when m divides k also x = fma(alpha_j, p_j, x) for
// j = k - m + 1 .. k ascending -- the x/r update's FMAs of variant 1, m
// iterations at a time.  Flush iterations take one element per thread per
// trip (m + 2 loads in flight).
__global__ void __launch_bounds__(kBlock) tri_pupdate_ring_kernel(int64_t n, const double *__restrict__ r,
                                                                 double *x, TriRing g,
                                                                 const TriScalars *sc) {
    pdl_wait();
    pdl_trigger();
    const double beta = ldg_o(&sc->slot[2]);
    const int k = ldg_o(&sc->it), m = g.m, R = m + 1;
    const double *src = tri_slot(g, (k - 1) % R);
    double *dst = tri_slot(g, k % R);
    const int64_t nth = gnth();
    if (k < 1) return;  // (max_iter 0: the body never runs)
    if (k % m != 0) {
        for (int64_t b0 = gtid(); b0 < n; b0 += kTriU * nth) {
            double pv[kTriU], rv[kTriU];
#pragma unroll
            for (int u = 0; u < kTriU; ++u) {
                const int64_t i = b0 + u * nth;
                if (i < n) {
                    pv[u] = src[i];
                    rv[u] = r[i];
                }
            }
#pragma unroll
            for (int u = 0; u < kTriU; ++u) {
                const int64_t i = b0 + u * nth;
                if (i < n) dst[i] = fma(beta, pv[u], rv[u]);
            }
        }
        return;
    }
    __shared__ const double *sop[kTriM];
    __shared__ double sal[kTriM];
    if (threadIdx.x < kTriM) {
        const int t = threadIdx.x, j = k - m + 1 + t;  // iterations k - m + 1 .. k
        sop[t] = t < m ? tri_slot(g, (j - 1) % R) : nullptr;
        sal[t] = t < m ? ldg_o(&sc->alpha_h[j & 15]) : 0.0;
    }
    __syncthreads();
    const double am = sal[m - 1];
    for (int64_t i = gtid(); i < n; i += nth) {
        double ov[kTriM - 1];
        const double rv = r[i], pk = src[i];  // p_k: the last direction (slot (k - 1) % R)
        double xv = x[i];
#pragma unroll
        for (int t = 0; t < kTriM - 1; ++t)
            if (t < m - 1) ov[t] = sop[t][i];
#pragma unroll
        for (int t = 0; t < kTriM - 1; ++t)
            if (t < m - 1) xv = fma(sal[t], ov[t], xv);
        x[i] = fma(am, pk, xv);
        dst[i] = fma(beta, pk, rv);
    }
}

// variant 2, after the loop: the directions since the last flush, j = F + 1
// .. N with F = m floor(N / m), N = it
__global__ void __launch_bounds__(kBlock) tri_xfix_kernel(int64_t n, double *x, TriRing g,
                                                         const TriScalars *sc) {
    pdl_wait();
    const int N = ldg_o(&sc->it), m = g.m, R = m + 1, F = m * (N / m), c = N - F;
    if (c == 0) return;
    __shared__ const double *sop[kTriM];
    __shared__ double sal[kTriM];
    if (threadIdx.x < kTriM) {
        const int t = threadIdx.x, j = F + 1 + t;
        sop[t] = t < c ? tri_slot(g, (j - 1) % R) : nullptr;
        sal[t] = t < c ? ldg_o(&sc->alpha_h[j & 15]) : 0.0;
    }
    __syncthreads();
    for (int64_t i = gtid(); i < n; i += gnth()) {
        double ov[kTriM];
#pragma unroll
        for (int t = 0; t < kTriM; ++t)
            if (t < c) ov[t] = sop[t][i];
        double xv = x[i];
#pragma unroll
        for (int t = 0; t < kTriM; ++t)
            if (t < c) xv = fma(sal[t], ov[t], xv);
        x[i] = xv;
    }
}

}  // namespace hpccg
