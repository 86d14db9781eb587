// spmvbench.cu -- SpMV kernel-design experiments on the 27-point ELL
// (slot-major, 128^3 by default), timed back to back on one GPU.  Not the
// product: the winner is ported into csrc/kernels.cuh.  Every variant must
// reproduce variant 0's bits (same FMA order).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o spmvbench spmvbench.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <vector>
#include <cooperative_groups.h>
namespace cgx = cooperative_groups;

constexpr int S = 27;

__device__ __forceinline__ uint64_t pol_ef() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ double lds(const double *p, uint64_t pol) {
    double v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int lds(const int *p, uint64_t pol) {
    int v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ double2 lds2(const double *p, uint64_t pol) {
    double2 v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;" : "=d"(v.x), "=d"(v.y) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int2 lds2(const int *p, uint64_t pol) {
    int2 v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.s32 {%0,%1}, [%2], %3;" : "=r"(v.x), "=r"(v.y) : "l"(p), "l"(pol));
    return v;
}

struct A {
    int64_t n, stride;
    const double *val;
    const int *col;
    const double *x;
    double *y;
};

// V0: product kernel (1 row / thread, groups of 9 slots)
template <int kBlk, int kMinB>
__global__ void __launch_bounds__(kBlk, kMinB) v0(A a) {
    const int64_t row = (int64_t)blockIdx.x * kBlk + threadIdx.x;
    if (row >= a.n) return;
    const uint64_t pol = pol_ef();
    double sum = 0.0;
#pragma unroll
    for (int g = 0; g < 3; ++g) {
        double vv[9];
        int cc[9];
#pragma unroll
        for (int t = 0; t < 9; ++t) {
            vv[t] = lds(a.val + (9 * g + t) * a.stride + row, pol);
            cc[t] = lds(a.col + (9 * g + t) * a.stride + row, pol);
        }
#pragma unroll
        for (int t = 0; t < 9; ++t) sum = fma(vv[t], __ldg(a.x + cc[t]), sum);
    }
    a.y[row] = sum;
}

// V1: all 54 loads first (no grouping)
template <int kBlk, int kMinB>
__global__ void __launch_bounds__(kBlk, kMinB) v1(A a) {
    const int64_t row = (int64_t)blockIdx.x * kBlk + threadIdx.x;
    if (row >= a.n) return;
    const uint64_t pol = pol_ef();
    double vv[S];
    int cc[S];
#pragma unroll
    for (int s = 0; s < S; ++s) {
        vv[s] = lds(a.val + s * a.stride + row, pol);
        cc[s] = lds(a.col + s * a.stride + row, pol);
    }
    double sum = 0.0;
#pragma unroll
    for (int s = 0; s < S; ++s) sum = fma(vv[s], __ldg(a.x + cc[s]), sum);
    a.y[row] = sum;
}

// V2: 2 rows / thread with 16-B val and 8-B col loads (n even)
template <int kBlk, int kMinB>
__global__ void __launch_bounds__(kBlk, kMinB) v2(A a) {
    const int64_t r2 = ((int64_t)blockIdx.x * kBlk + threadIdx.x) * 2;
    if (r2 >= a.n) return;
    const uint64_t pol = pol_ef();
    double s0 = 0.0, s1 = 0.0;
#pragma unroll
    for (int g = 0; g < 3; ++g) {
        double2 vv[9];
        int2 cc[9];
#pragma unroll
        for (int t = 0; t < 9; ++t) {
            vv[t] = lds2(a.val + (9 * g + t) * a.stride + r2, pol);
            cc[t] = lds2(a.col + (9 * g + t) * a.stride + r2, pol);
        }
#pragma unroll
        for (int t = 0; t < 9; ++t) {
            s0 = fma(vv[t].x, __ldg(a.x + cc[t].x), s0);
            s1 = fma(vv[t].y, __ldg(a.x + cc[t].y), s1);
        }
    }
    *reinterpret_cast<double2 *>(a.y + r2) = make_double2(s0, s1);
}

// V3: persistent grid-stride over 1-row-per-thread tiles
template <int kBlk, int kMinB>
__global__ void __launch_bounds__(kBlk, kMinB) v3(A a) {
    const uint64_t pol = pol_ef();
    for (int64_t row = (int64_t)blockIdx.x * kBlk + threadIdx.x; row < a.n; row += (int64_t)gridDim.x * kBlk) {
        double sum = 0.0;
#pragma unroll
        for (int g = 0; g < 3; ++g) {
            double vv[9];
            int cc[9];
#pragma unroll
            for (int t = 0; t < 9; ++t) {
                vv[t] = lds(a.val + (9 * g + t) * a.stride + row, pol);
                cc[t] = lds(a.col + (9 * g + t) * a.stride + row, pol);
            }
#pragma unroll
            for (int t = 0; t < 9; ++t) sum = fma(vv[t], __ldg(a.x + cc[t]), sum);
        }
        a.y[row] = sum;
    }
}

// V4: 2 rows / thread, groups of 3 slots (lower register use, more threads)
template <int kBlk, int kMinB>
__global__ void __launch_bounds__(kBlk, kMinB) v4(A a) {
    const int64_t r2 = ((int64_t)blockIdx.x * kBlk + threadIdx.x) * 2;
    if (r2 >= a.n) return;
    const uint64_t pol = pol_ef();
    double s0 = 0.0, s1 = 0.0;
#pragma unroll
    for (int g = 0; g < 9; ++g) {
        double2 vv[3];
        int2 cc[3];
#pragma unroll
        for (int t = 0; t < 3; ++t) {
            vv[t] = lds2(a.val + (3 * g + t) * a.stride + r2, pol);
            cc[t] = lds2(a.col + (3 * g + t) * a.stride + r2, pol);
        }
#pragma unroll
        for (int t = 0; t < 3; ++t) {
            s0 = fma(vv[t].x, __ldg(a.x + cc[t].x), s0);
            s1 = fma(vv[t].y, __ldg(a.x + cc[t].y), s1);
        }
    }
    *reinterpret_cast<double2 *>(a.y + r2) = make_double2(s0, s1);
}

// V5 / V6: the north_star's "shared-memory or TMA staging of x-planes".  A CTA
// of 256 threads owns 512 rows [r0, r0 + 512) (2 rows / thread, the v4 matrix
// stream); the x entries those rows can touch lie in three windows (z - 1,
// z, z + 1 planes: r0 + (dz + 1) plane - (nx + 1) ... + 512 + nx + 1), staged
// into shared memory -- V5 by three 1-D TMA bulk copies (cp.async.bulk, one
// mbarrier, issued by one thread while every thread starts its matrix loads),
// V6 by the CTA's threads (coalesced loads + __syncthreads).  Gathers take
// slot s's window (s / 9, the generator's sz-major slot order) as a hint and
// fall back to a global load when the column lies outside it, so any matrix
// stays correct.  Same FMA order as v0: identical bits.
struct StageArgs {
    int64_t plane, ncol;
    int nx, wmax;  // wmax: doubles per staged window (even)
};

__device__ __forceinline__ void stage_window(const A &a, const StageArgs &g, int64_t r0, int w,
                                             int64_t &lo, int &len) {
    int64_t b = r0 + (int64_t)w * g.plane - (g.nx + 1);  // local-with-halo index of the window start
    int64_t e = r0 + (int64_t)w * g.plane + 512 + g.nx + 1;
    b = b < 0 ? 0 : (b & ~(int64_t)1);                   // 16-B aligned start
    e = e > g.ncol ? g.ncol : ((e + 1) & ~(int64_t)1);
    lo = b;
    len = (int)(e - b);
    if (len > g.wmax) len = g.wmax;
}

template <bool kTma>
__global__ void __launch_bounds__(256, 3) v56(A a, StageArgs g) {
    extern __shared__ __align__(16) double xs[];
    __shared__ __align__(8) unsigned long long mbar;
    const int64_t r0 = (int64_t)blockIdx.x * 512;
    int64_t lo[3];
    int len[3];
#pragma unroll
    for (int w = 0; w < 3; ++w) stage_window(a, g, r0, w, lo[w], len[w]);
    const unsigned mb = (unsigned)__cvta_generic_to_shared(&mbar);
    if (kTma) {
        if (threadIdx.x == 0) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb));
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
            const unsigned tx = (unsigned)(8 * (len[0] + len[1] + len[2]));
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(tx) : "memory");
#pragma unroll
            for (int w = 0; w < 3; ++w) {
                const unsigned dst = (unsigned)__cvta_generic_to_shared(xs + w * g.wmax);
                asm volatile(
                    "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                    "l"(a.x + lo[w]), "r"((unsigned)(8 * len[w])), "r"(mb)
                    : "memory");
            }
        }
    } else {
        for (int w = 0; w < 3; ++w)
            for (int i = threadIdx.x; i < len[w]; i += 256) xs[w * g.wmax + i] = __ldg(a.x + lo[w] + i);
    }
    const int64_t r2 = r0 + 2 * threadIdx.x;
    const uint64_t pol = pol_ef();
    double s0 = 0.0, s1 = 0.0;
    const bool live = r2 < a.n;
#pragma unroll
    for (int gi = 0; gi < 9; ++gi) {
        double2 vv[3];
        int2 cc[3];
        if (live) {
#pragma unroll
            for (int t = 0; t < 3; ++t) {
                vv[t] = lds2(a.val + (3 * gi + t) * a.stride + r2, pol);
                cc[t] = lds2(a.col + (3 * gi + t) * a.stride + r2, pol);
            }
        }
        if (gi == 0) {  // the staged windows are needed from here on
            if (kTma) {
                __syncthreads();  // mbarrier initialised before anyone waits on it
                unsigned ok = 0;
                while (!ok)
                    asm volatile(
                        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
                        : "=r"(ok) : "r"(mb) : "memory");
            } else {
                __syncthreads();
            }
        }
        if (live) {
#pragma unroll
            for (int t = 0; t < 3; ++t) {
                const int w = (3 * gi + t) / 9;
                const int64_t o0 = (int64_t)cc[t].x - lo[w], o1 = (int64_t)cc[t].y - lo[w];
                const double xa = (uint64_t)o0 < (uint64_t)len[w] ? xs[w * g.wmax + o0] : __ldg(a.x + cc[t].x);
                const double xb = (uint64_t)o1 < (uint64_t)len[w] ? xs[w * g.wmax + o1] : __ldg(a.x + cc[t].y);
                s0 = fma(vv[t].x, xa, s0);
                s1 = fma(vv[t].y, xb, s1);
            }
        }
    }
    if (live) *reinterpret_cast<double2 *>(a.y + r2) = make_double2(s0, s1);
}

struct Red {
    double *partials;
    unsigned *counter;
    double *out;
    const int *done;
};

__device__ __forceinline__ double wsum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

__device__ __forceinline__ unsigned n_partials_base(unsigned nb) { return (nb + 31) / 32 * 32; }

// kMode: 0 partial store only, 1 fence + atomicAdd + last block, 2 red.release + last block
template <int kMode, bool kCheck>
__global__ void __launch_bounds__(256, 4) vdot(A a, Red red) {
    const int64_t row = (int64_t)blockIdx.x * 256 + threadIdx.x;
    const uint64_t pol = pol_ef();
    double d = 0.0;
    const int done = kCheck ? __ldg(red.done) : 0;
    if (row < a.n) {
        double sum = 0.0, xd = 0.0;
#pragma unroll
        for (int g = 0; g < 3; ++g) {
            double vv[9];
            int cc[9];
#pragma unroll
            for (int t = 0; t < 9; ++t) {
                vv[t] = lds(a.val + (9 * g + t) * a.stride + row, pol);
                cc[t] = lds(a.col + (9 * g + t) * a.stride + row, pol);
            }
            if (g == 0 && done) return;
#pragma unroll
            for (int t = 0; t < 9; ++t) {
                const double xv = __ldg(a.x + cc[t]);
                if (9 * g + t == 13) xd = xv;
                sum = fma(vv[t], xv, sum);
            }
        }
        a.y[row] = sum;
        d = sum * xd;
    }
    __shared__ double sh[8];
    __shared__ int last;
    d = wsum(d);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = d;
    __syncthreads();
    if (threadIdx.x < 32) {
        d = threadIdx.x < 8 ? sh[threadIdx.x] : 0.0;
        d = wsum(d);
        if (threadIdx.x == 0) {
            red.partials[blockIdx.x] = d;
            if (kMode == 1) {
                __threadfence();
                last = atomicAdd(red.counter, 1u) == gridDim.x - 1;
            } else if (kMode == 2) {
                unsigned t;
                asm volatile("atom.add.release.gpu.u32 %0, [%1], 1;" : "=r"(t) : "l"(red.counter) : "memory");
                last = t == gridDim.x - 1;
            } else if (kMode == 3) {
                __threadfence();
                last = 0;
            } else if (kMode == 4) {
                // hierarchical: group counters (64 blocks each), then a top counter
                __threadfence();
                const unsigned g = blockIdx.x / 64, ng = (gridDim.x + 63) / 64;
                const unsigned gsz = min(64u, gridDim.x - g * 64);
                last = 0;
                if (atomicAdd(red.counter + 32 * (1 + g), 1u) == gsz - 1) {
                    __threadfence();
                    double gs = 0.0;
                    for (unsigned i = 0; i < gsz; ++i) gs += __ldcg(red.partials + g * 64 + i);
                    red.partials[(n_partials_base(gridDim.x)) + g] = gs;
                    red.counter[32 * (1 + g)] = 0;
                    __threadfence();
                    last = atomicAdd(red.counter, 1u) == ng - 1 ? 2 : 0;
                }
            } else if (kMode == 5) {
                // 32 strided arrival counters (blocks b = j mod 32 share counter j), then a top counter
                __threadfence();
                const unsigned j = blockIdx.x & 31;
                const unsigned cnt = (gridDim.x - j + 31) / 32;
                last = 0;
                if (atomicAdd(red.counter + 32 * (1 + j), 1u) == cnt - 1) {
                    red.counter[32 * (1 + j)] = 0;
                    last = atomicAdd(red.counter, 1u) == 31;
                }
            } else {
                last = 0;
            }
        }
    }
    __syncthreads();
    if (!last) return;
    if (kMode == 4) {
        if (threadIdx.x == 0) {
            __threadfence();
            const unsigned ng = (gridDim.x + 63) / 64;
            double s = 0.0;
            for (unsigned i = 0; i < ng; ++i) s += __ldcg(red.partials + n_partials_base(gridDim.x) + i);
            *red.counter = 0;
            *red.out = s;
        }
        return;
    }
    if (kMode == 2) asm volatile("fence.acq_rel.gpu;" ::: "memory");
    else __threadfence();
    double s = 0.0;
    for (unsigned i = threadIdx.x; i < gridDim.x; i += 256) s += __ldcg(red.partials + i);
    s = wsum(s);
    __syncthreads();
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x < 32) {
        s = threadIdx.x < 8 ? sh[threadIdx.x] : 0.0;
        s = wsum(s);
        if (threadIdx.x == 0) {
            *red.counter = 0;
            *red.out = s;
        }
    }
}

// 2 rows / thread (16-B val, 8-B col loads), groups of 3 slots, p.Ap epilogue
// with the fence + atomic last-block finisher; kBlk threads -> 2 kBlk rows.
template <int kBlk, int kMinB>
__global__ void __launch_bounds__(kBlk, kMinB) vdot2(A a, Red red) {
    const int64_t r2 = ((int64_t)blockIdx.x * kBlk + threadIdx.x) * 2;
    const uint64_t pol = pol_ef();
    double d = 0.0;
    if (r2 < a.n) {
        double s0 = 0.0, s1 = 0.0, x0 = 0.0, x1 = 0.0;
#pragma unroll
        for (int g = 0; g < 9; ++g) {
            double2 vv[3];
            int2 cc[3];
#pragma unroll
            for (int t = 0; t < 3; ++t) {
                vv[t] = lds2(a.val + (3 * g + t) * a.stride + r2, pol);
                cc[t] = lds2(a.col + (3 * g + t) * a.stride + r2, pol);
            }
#pragma unroll
            for (int t = 0; t < 3; ++t) {
                const double xa = __ldg(a.x + cc[t].x), xb = __ldg(a.x + cc[t].y);
                if (3 * g + t == 13) { x0 = xa; x1 = xb; }
                s0 = fma(vv[t].x, xa, s0);
                s1 = fma(vv[t].y, xb, s1);
            }
        }
        *reinterpret_cast<double2 *>(a.y + r2) = make_double2(s0, s1);
        d = fma(s1, x1, s0 * x0);
    }
    constexpr int W = kBlk / 32;
    __shared__ double sh[32];
    __shared__ int last;
    d = wsum(d);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = d;
    __syncthreads();
    if (threadIdx.x < 32) {
        d = threadIdx.x < W ? sh[threadIdx.x] : 0.0;
        d = wsum(d);
        if (threadIdx.x == 0) {
            red.partials[blockIdx.x] = d;
            __threadfence();
            last = atomicAdd(red.counter, 1u) == gridDim.x - 1;
        }
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    double s = 0.0;
    for (unsigned i = threadIdx.x; i < gridDim.x; i += kBlk) s += __ldcg(red.partials + i);
    s = wsum(s);
    __syncthreads();
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x < 32) {
        s = threadIdx.x < W ? sh[threadIdx.x] : 0.0;
        s = wsum(s);
        if (threadIdx.x == 0) {
            *red.counter = 0;
            *red.out = s;
        }
    }
}

// 2 rows / thread + p.Ap with a CLUSTER-level pre-reduction: the 8 CTAs of a
// cluster hand their partials to CTA 0 through DSMEM (+ a DSMEM atomic
// arrival count); only CTA 0 does the global fence + ticket.
template <int kCl>
__global__ void __launch_bounds__(256, 4) vdot2c(A a, Red red) {
    auto cluster = cgx::this_cluster();
    __shared__ double cl_part[kCl];
    __shared__ unsigned cl_count;
    const unsigned crank = cluster.block_rank();
    if (threadIdx.x == 0) cl_count = 0;
    cluster.sync();  // CTA 0's counter initialised before anyone arrives
    const int64_t r2 = ((int64_t)blockIdx.x * 256 + threadIdx.x) * 2;
    const uint64_t pol = pol_ef();
    double d = 0.0;
    if (r2 < a.n) {
        double s0 = 0.0, s1 = 0.0, x0 = 0.0, x1 = 0.0;
#pragma unroll
        for (int g = 0; g < 9; ++g) {
            double2 vv[3];
            int2 cc[3];
#pragma unroll
            for (int t = 0; t < 3; ++t) {
                vv[t] = lds2(a.val + (3 * g + t) * a.stride + r2, pol);
                cc[t] = lds2(a.col + (3 * g + t) * a.stride + r2, pol);
            }
#pragma unroll
            for (int t = 0; t < 3; ++t) {
                const double xa = __ldg(a.x + cc[t].x), xb = __ldg(a.x + cc[t].y);
                if (3 * g + t == 13) { x0 = xa; x1 = xb; }
                s0 = fma(vv[t].x, xa, s0);
                s1 = fma(vv[t].y, xb, s1);
            }
        }
        *reinterpret_cast<double2 *>(a.y + r2) = make_double2(s0, s1);
        d = fma(s1, x1, s0 * x0);
    }
    __shared__ double sh[32];
    __shared__ int last;
    d = wsum(d);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = d;
    __syncthreads();
    if (threadIdx.x < 32) {
        d = threadIdx.x < 8 ? sh[threadIdx.x] : 0.0;
        d = wsum(d);
    }
    if (crank != 0) {
        if (threadIdx.x == 0) {
            double *rp = cluster.map_shared_rank(cl_part, 0);
            unsigned *rc = cluster.map_shared_rank(&cl_count, 0);
            rp[crank] = d;
            asm volatile("red.release.cluster.add.u32 [%0], 1;" ::"l"(rc) : "memory");
        }
        return;
    }
    if (threadIdx.x == 0) {
        cl_part[0] = d;
        unsigned c;
        do {
            asm volatile("ld.acquire.cluster.u32 %0, [%1];" : "=r"(c) : "l"(&cl_count) : "memory");
        } while (c != kCl - 1);
        double cs = 0.0;
        for (int k = 0; k < kCl; ++k) cs += cl_part[k];
        const unsigned ncl = gridDim.x / kCl;
        red.partials[blockIdx.x / kCl] = cs;
        __threadfence();
        last = atomicAdd(red.counter, 1u) == ncl - 1;
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    const unsigned ncl = gridDim.x / kCl;
    double s = 0.0;
    for (unsigned i = threadIdx.x; i < ncl; i += 256) s += __ldcg(red.partials + i);
    s = wsum(s);
    __syncthreads();
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x < 32) {
        s = threadIdx.x < 8 ? sh[threadIdx.x] : 0.0;
        s = wsum(s);
        if (threadIdx.x == 0) {
            *red.counter = 0;
            *red.out = s;
        }
    }
}

template <int kCl>
void launch_vdot2c(A a, Red red, int64_t n) {
    const unsigned blocks = (unsigned)(((n / 2 + 255) / 256 + kCl - 1) / kCl * kCl);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(blocks);
    cfg.blockDim = dim3(256);
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = kCl;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, vdot2c<kCl>, a, red);
    if (e != cudaSuccess) printf("launch error %s\n", cudaGetErrorString(e));
}

template <class F>
float timeit(F f, int reps) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    f();
    cudaDeviceSynchronize();
    cudaEventRecord(e0);
    for (int r = 0; r < reps; ++r) f();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    return ms / reps;
}

int main(int argc, char **argv) {
    const int nx = argc > 1 ? atoi(argv[1]) : 128, ny = argc > 2 ? atoi(argv[2]) : 128,
              nz = argc > 3 ? atoi(argv[3]) : 128;
    const int64_t plane = (int64_t)nx * ny, n = plane * nz, ncol = n + 2 * plane;
    std::vector<double> hv((size_t)S * n);
    std::vector<int> hc((size_t)S * n);
    int64_t nnz = 0;
    for (int64_t i = 0; i < n; ++i) {
        const int64_t iz = i / plane, iy = (i % plane) / nx, ix = i % nx;
        for (int s = 0; s < S; ++s) {
            const int sz = s / 9 - 1, sy = (s / 3) % 3 - 1, sx = s % 3 - 1;
            const bool in = ix + sx >= 0 && ix + sx < nx && iy + sy >= 0 && iy + sy < ny && iz + sz >= 0 && iz + sz < nz;
            hv[(size_t)s * n + i] = in ? (s == 13 ? 27.0 : -1.0) : 0.0;
            hc[(size_t)s * n + i] = (int)(i + plane + (in ? sz * plane + sy * nx + sx : 0));
            nnz += in;
        }
    }
    std::vector<double> hx(ncol);
    for (int64_t j = 0; j < ncol; ++j) hx[j] = (double)((j * 2654435761ull) % 1000) / 997.0 - 0.5;
    double *val, *x, *y, *yref;
    int *col;
    cudaMalloc(&val, sizeof(double) * S * n);
    cudaMalloc(&col, sizeof(int) * S * n);
    cudaMalloc(&x, sizeof(double) * ncol);
    cudaMalloc(&y, sizeof(double) * n);
    cudaMalloc(&yref, sizeof(double) * n);
    cudaMemcpy(val, hv.data(), sizeof(double) * S * n, cudaMemcpyHostToDevice);
    cudaMemcpy(col, hc.data(), sizeof(int) * S * n, cudaMemcpyHostToDevice);
    cudaMemcpy(x, hx.data(), sizeof(double) * ncol, cudaMemcpyHostToDevice);
    A a{n, n, val, col, x, yref};
    const double alg = 12.0 * nnz + 16.0 * n;
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    v0<256, 4><<<(unsigned)((n + 255) / 256), 256>>>(a);
    cudaDeviceSynchronize();
    std::vector<double> ref(n), got(n);
    cudaMemcpy(ref.data(), yref, sizeof(double) * n, cudaMemcpyDeviceToHost);
    a.y = y;
    auto report = [&](const char *name, float ms) {
        cudaMemcpy(got.data(), y, sizeof(double) * n, cudaMemcpyDeviceToHost);
        const bool ok = memcmp(got.data(), ref.data(), sizeof(double) * n) == 0;
        cudaMemset(y, 0, sizeof(double) * n);
        printf("{\"variant\": \"%s\", \"us\": %.2f, \"alg_GBs\": %.1f, \"bitwise\": %s}\n", name, ms * 1e3,
               alg / (ms * 1e-3) / 1e9, ok ? "true" : "false");
        fflush(stdout);
    };
    const int R = 30;
    const unsigned g256 = (unsigned)((n + 255) / 256), g128 = (unsigned)((n + 127) / 128);
#define RUN(NAME, ...) report(NAME, timeit([&] { __VA_ARGS__; }, R))
    RUN("v0_b256_m4", (v0<256, 4><<<g256, 256>>>(a)));
    RUN("v0_b256_m3", (v0<256, 3><<<g256, 256>>>(a)));
    RUN("v0_b256_m5", (v0<256, 5><<<g256, 256>>>(a)));
    RUN("v0_b256_m6", (v0<256, 6><<<g256, 256>>>(a)));
    RUN("v0_b128_m8", (v0<128, 8><<<g128, 128>>>(a)));
    RUN("v0_b128_m12", (v0<128, 12><<<g128, 128>>>(a)));
    RUN("v0_b512_m2", (v0<512, 2><<<(unsigned)((n + 511) / 512), 512>>>(a)));
    RUN("v1_b256_m2", (v1<256, 2><<<g256, 256>>>(a)));
    RUN("v1_b256_m3", (v1<256, 3><<<g256, 256>>>(a)));
    RUN("v2_b128_m4", (v2<128, 4><<<(unsigned)((n / 2 + 127) / 128), 128>>>(a)));
    RUN("v2_b128_m6", (v2<128, 6><<<(unsigned)((n / 2 + 127) / 128), 128>>>(a)));
    RUN("v2_b256_m2", (v2<256, 2><<<(unsigned)((n / 2 + 255) / 256), 256>>>(a)));
    RUN("v2_b256_m3", (v2<256, 3><<<(unsigned)((n / 2 + 255) / 256), 256>>>(a)));
    RUN("v4_b128_m8", (v4<128, 8><<<(unsigned)((n / 2 + 127) / 128), 128>>>(a)));
    RUN("v4_b256_m4", (v4<256, 4><<<(unsigned)((n / 2 + 255) / 256), 256>>>(a)));
    RUN("v4_b256_m6", (v4<256, 6><<<(unsigned)((n / 2 + 255) / 256), 256>>>(a)));
    Red red;
    cudaMalloc(&red.partials, sizeof(double) * (2 * (n / 256) + 4096));
    cudaMalloc(&red.counter, 4 * 32 * 4096);
    cudaMemset(red.counter, 0, 4 * 32 * 4096);
    cudaMalloc(&red.out, 64);
    cudaMalloc((void **)&red.done, 64);
    cudaMemset(red.counter, 0, 64);
    cudaMemset((void *)red.done, 0, 64);
    RUN("vdot_partials_only", (vdot<0, false><<<g256, 256>>>(a, red)));
    RUN("vdot_fence_atomic", (vdot<1, false><<<g256, 256>>>(a, red)));
    RUN("vdot_release_atomic", (vdot<2, false><<<g256, 256>>>(a, red)));
    RUN("vdot_fence_only", (vdot<3, false><<<g256, 256>>>(a, red)));
    RUN("vdot_hier64", (vdot<4, false><<<g256, 256>>>(a, red)));
    RUN("vdot_strided32", (vdot<5, false><<<g256, 256>>>(a, red)));
    RUN("vdot_strided32_check", (vdot<5, true><<<g256, 256>>>(a, red)));
    RUN("vdot_fence_atomic_check", (vdot<1, true><<<g256, 256>>>(a, red)));
    RUN("vdot_release_atomic_check", (vdot<2, true><<<g256, 256>>>(a, red)));
    RUN("vdot2_b128_m8", (vdot2<128, 8><<<(unsigned)((n / 2 + 127) / 128), 128>>>(a, red)));
    RUN("vdot2_b256_m4", (vdot2<256, 4><<<(unsigned)((n / 2 + 255) / 256), 256>>>(a, red)));
    RUN("vdot2_b512_m2", (vdot2<512, 2><<<(unsigned)((n / 2 + 511) / 512), 512>>>(a, red)));
    RUN("vdot2_b1024_m1", (vdot2<1024, 1><<<(unsigned)((n / 2 + 1023) / 1024), 1024>>>(a, red)));
    RUN("vdot2c_cl2", (launch_vdot2c<2>(a, red, n)));
    RUN("vdot2c_cl4", (launch_vdot2c<4>(a, red, n)));
    RUN("vdot2c_cl8", (launch_vdot2c<8>(a, red, n)));
    {
        double h_out;
        cudaMemcpy(&h_out, red.out, 8, cudaMemcpyDeviceToHost);
        launch_vdot2c<8>(a, red, n);
        double h2;
        cudaDeviceSynchronize();
        cudaMemcpy(&h2, red.out, 8, cudaMemcpyDeviceToHost);
        vdot2<256, 4><<<(unsigned)((n / 2 + 255) / 256), 256>>>(a, red);
        double h3;
        cudaDeviceSynchronize();
        cudaMemcpy(&h3, red.out, 8, cudaMemcpyDeviceToHost);
        printf("{\"dot_cluster8\": %.17g, \"dot_flat\": %.17g, \"rel\": %.3g, \"err\": \"%s\"}\n", h2, h3,
               (h2 - h3) / h3, cudaGetErrorString(cudaGetLastError()));
    }
    RUN("v0_b256_m4_again", (v0<256, 4><<<g256, 256>>>(a)));
    {   // x-plane staging (north_star): TMA bulk copies vs cooperative loads, vs v4
        StageArgs sg{plane, ncol, nx, (512 + 2 * (nx + 1) + 4) & ~1};
        const size_t sm = sizeof(double) * 3 * sg.wmax;
        cudaFuncSetAttribute(v56<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        cudaFuncSetAttribute(v56<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        const unsigned g512 = (unsigned)((n + 511) / 512);
        for (int rep = 0; rep < 2; ++rep) {
            RUN("v4_b256_m4_ref", (v4<256, 4><<<(unsigned)((n / 2 + 255) / 256), 256>>>(a)));
            RUN("v5_tma_staged_x", (v56<true><<<g512, 256, sm>>>(a, sg)));
            RUN("v6_smem_staged_x", (v56<false><<<g512, 256, sm>>>(a, sg)));
        }
        printf("{\"staged_window_doubles\": %d, \"smem_bytes\": %zu, \"err\": \"%s\"}\n", sg.wmax, sm,
               cudaGetErrorString(cudaGetLastError()));
    }
    for (int w : {1, 2, 4}) {
        int occ;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, v3<256, 4>, 256, 0);
        char nm[64];
        snprintf(nm, sizeof nm, "v3_persist_w%d", w);
        RUN(nm, (v3<256, 4><<<(unsigned)(sms * occ * w), 256>>>(a)));
    }
    return 0;
}
