// tmaspmv.cu -- experiment: the 27-point ELL SpMV with the MATRIX STREAM fed by
// TMA bulk copies into a shared-memory ring (persistent CTAs, static
// interleaved chunks) vs the product's per-thread-load kernel (2 rows per
// thread, groups of 3 slots).  Same per-row FMA chain (ascending slot), so y
// must be bitwise identical.  Not the product.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tmaspmv tmaspmv.cu
//   ./tmaspmv [nx ny nz]
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <vector>

constexpr int S = 27;

__device__ __forceinline__ uint64_t pol_ef() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
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
    int64_t n, plane;
    int nx, ny;
    double *val;
    int *col;
    const double *x;
    double *y;
};

__global__ void gen(A a) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= a.n) return;
    const int64_t nz = a.n / a.plane;
    const int64_t iz = i / a.plane, iy = (i % a.plane) / a.nx, ix = i % a.nx;
    for (int s = 0; s < S; ++s) {
        const int sz = s / 9 - 1, sy = (s / 3) % 3 - 1, sx = s % 3 - 1;
        const bool in = ix + sx >= 0 && ix + sx < a.nx && iy + sy >= 0 && iy + sy < a.ny && iz + sz >= 0 && iz + sz < nz;
        a.val[(int64_t)s * a.n + i] = in ? (s == 13 ? 27.0 : -1.0) : 0.0;
        a.col[(int64_t)s * a.n + i] = (int)(i + a.plane + (in ? sz * a.plane + sy * a.nx + sx : 0));
    }
}

__global__ void xinit(double *x, int64_t m) {
    const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < m) x[j] = (double)((j * 2654435761ull) % 1000) / 997.0 - 0.5;
}

// the product kernel's structure: 2 rows / thread, groups of 3 slots
__global__ void __launch_bounds__(256, 4) ref(A a) {
    const int64_t r2 = ((int64_t)blockIdx.x * 256 + threadIdx.x) * 2;
    if (r2 >= a.n) return;
    const uint64_t pol = pol_ef();
    double s0 = 0.0, s1 = 0.0;
#pragma unroll
    for (int g = 0; g < 9; ++g) {
        double2 vv[3];
        int2 cc[3];
#pragma unroll
        for (int t = 0; t < 3; ++t) {
            vv[t] = lds2(a.val + (3 * g + t) * a.n + r2, pol);
            cc[t] = lds2(a.col + (3 * g + t) * a.n + r2, pol);
        }
#pragma unroll
        for (int t = 0; t < 3; ++t) {
            s0 = fma(vv[t].x, __ldg(a.x + cc[t].x), s0);
            s1 = fma(vv[t].y, __ldg(a.x + cc[t].y), s1);
        }
    }
    *reinterpret_cast<double2 *>(a.y + r2) = make_double2(s0, s1);
}

// TMA-fed: persistent CTA, chunks of R rows (c = blockIdx.x + i * gridDim.x),
// a ring of KS stages; stage layout: val[27][R] doubles, col[27][R] ints.
// Thread 0 issues the 54 bulk copies of a chunk (one per slot and array) on
// the stage's mbarrier; NT threads compute R rows (2 rows per thread per pass).
template <int R, int KS, int NT>
__global__ void __launch_bounds__(NT, 1) tma(A a) {
    extern __shared__ __align__(128) unsigned char ring[];
    __shared__ __align__(8) unsigned long long full[KS];
    constexpr int kStage = R * S * 12;
    const int64_t nch = (a.n + R - 1) / R;
    const int64_t mine = blockIdx.x < nch ? (nch - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    auto issue = [&](int64_t i, int s) {
        const int64_t c = blockIdx.x + i * gridDim.x;
        const int64_t r0 = c * R;
        const int rows = (int)((a.n - r0) < R ? (a.n - r0) : R);
        const unsigned mb = (unsigned)__cvta_generic_to_shared(&full[s]);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"((unsigned)(rows * S * 12)) : "memory");
        unsigned char *st = ring + (size_t)s * kStage;
        for (int k = 0; k < S; ++k) {
            const unsigned dv = (unsigned)__cvta_generic_to_shared(st + (size_t)k * R * 8);
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(dv), "l"(a.val + (int64_t)k * a.n + r0), "r"((unsigned)(rows * 8)), "r"(mb) : "memory");
            const unsigned dc = (unsigned)__cvta_generic_to_shared(st + (size_t)S * R * 8 + (size_t)k * R * 4);
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(dc), "l"(a.col + (int64_t)k * a.n + r0), "r"((unsigned)(rows * 4)), "r"(mb) : "memory");
        }
    };
    if (threadIdx.x == 0) {
        for (int s = 0; s < KS; ++s) {
            const unsigned mb = (unsigned)__cvta_generic_to_shared(&full[s]);
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int s = 0; s < KS && s < mine; ++s) issue(s, s);
    }
    __syncthreads();
    for (int64_t i = 0; i < mine; ++i) {
        const int s = (int)(i % KS);
        const unsigned par = (unsigned)((i / KS) & 1);
        const unsigned mb = (unsigned)__cvta_generic_to_shared(&full[s]);
        unsigned ok = 0;
        while (!ok)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                         : "=r"(ok) : "r"(mb), "r"(par) : "memory");
        const unsigned char *st = ring + (size_t)s * kStage;
        const double *sv = reinterpret_cast<const double *>(st);
        const int *sc = reinterpret_cast<const int *>(st + (size_t)S * R * 8);
        const int64_t r0 = (blockIdx.x + i * gridDim.x) * R;
        for (int j = 2 * threadIdx.x; j < R; j += 2 * NT) {
            const int64_t r2 = r0 + j;
            if (r2 >= a.n) break;
            double s0 = 0.0, s1 = 0.0;
            double2 xv[S];
#pragma unroll
            for (int k = 0; k < S; ++k) {  // all 54 gathers in flight
                const int2 cc = *reinterpret_cast<const int2 *>(sc + k * R + j);
                xv[k] = make_double2(__ldg(a.x + cc.x), __ldg(a.x + cc.y));
            }
#pragma unroll
            for (int k = 0; k < S; ++k) {
                const double2 vv = *reinterpret_cast<const double2 *>(sv + k * R + j);
                s0 = fma(vv.x, xv[k].x, s0);
                s1 = fma(vv.y, xv[k].y, s1);
            }
            *reinterpret_cast<double2 *>(a.y + r2) = make_double2(s0, s1);
        }
        __syncthreads();  // stage s consumed
        if (threadIdx.x == 0 && i + KS < mine) issue(i + KS, s);
    }
}

template <class F>
float best_ms(F f, int reps) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    f();
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int r = 0; r < reps; ++r) {
        cudaEventRecord(e0);
        f();
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        best = ms < best ? ms : best;
    }
    return best;
}

// Sliced copy of the same ELL: chunk c of R rows stored contiguously as
// val[27][R] doubles then col[27][R] ints (R * 324 B); built once from the
// slot-major arrays.  Rows past n in the last chunk are padding (val 0, col of
// row 0's diagonal).
template <int R>
__global__ void make_sliced(A a, unsigned char *sl) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nch = (a.n + R - 1) / R;
    if (i >= nch * R) return;
    const int64_t c = i / R, j = i % R;
    double *v = reinterpret_cast<double *>(sl + (size_t)c * R * 324);
    int *cc = reinterpret_cast<int *>(sl + (size_t)c * R * 324 + (size_t)R * 27 * 8);
    for (int k = 0; k < S; ++k) {
        v[k * R + j] = i < a.n ? a.val[(int64_t)k * a.n + i] : 0.0;
        cc[k * R + j] = i < a.n ? a.col[(int64_t)k * a.n + i] : (int)a.plane;
    }
}

// TMA-fed over the sliced copy: ONE bulk copy per chunk (R * 324 B), KS-stage
// ring, persistent CTAs with static interleaved chunks, kRows rows per thread.
template <int R, int KS, int NT>
__global__ void __launch_bounds__(NT, 1) tma_sliced(A a, const unsigned char *sl) {
    extern __shared__ __align__(128) unsigned char ring[];
    __shared__ __align__(8) unsigned long long full[KS];
    constexpr unsigned kStage = R * 324;
    constexpr int kRows = R / NT;  // rows per thread per chunk (1 or 2)
    const int64_t nch = (a.n + R - 1) / R;
    const int64_t mine = blockIdx.x < nch ? (nch - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    auto issue = [&](int64_t i, int s) {
        const int64_t c = blockIdx.x + i * gridDim.x;
        const unsigned mb = (unsigned)__cvta_generic_to_shared(&full[s]);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(kStage) : "memory");
        const unsigned dst = (unsigned)__cvta_generic_to_shared(ring + (size_t)s * kStage);
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(dst), "l"(sl + (size_t)c * kStage), "r"(kStage), "r"(mb) : "memory");
    };
    if (threadIdx.x == 0) {
        for (int s = 0; s < KS; ++s) {
            const unsigned mb = (unsigned)__cvta_generic_to_shared(&full[s]);
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int s = 0; s < KS && s < mine; ++s) issue(s, s);
    }
    __syncthreads();
    for (int64_t i = 0; i < mine; ++i) {
        const int s = (int)(i % KS);
        const unsigned par = (unsigned)((i / KS) & 1);
        const unsigned mb = (unsigned)__cvta_generic_to_shared(&full[s]);
        unsigned ok = 0;
        while (!ok)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                         : "=r"(ok) : "r"(mb), "r"(par) : "memory");
        const unsigned char *st = ring + (size_t)s * kStage;
        const double *sv = reinterpret_cast<const double *>(st);
        const int *sc = reinterpret_cast<const int *>(st + (size_t)S * R * 8);
        const int64_t r0 = (blockIdx.x + i * gridDim.x) * R;
        if (kRows == 2) {
            const int j = 2 * threadIdx.x;
            const int64_t r2 = r0 + j;
            double2 xv[S];
#pragma unroll
            for (int k = 0; k < S; ++k) {
                const int2 cc = *reinterpret_cast<const int2 *>(sc + k * R + j);
                xv[k] = make_double2(__ldg(a.x + cc.x), __ldg(a.x + cc.y));
            }
            double s0 = 0.0, s1 = 0.0;
#pragma unroll
            for (int k = 0; k < S; ++k) {
                const double2 vv = *reinterpret_cast<const double2 *>(sv + k * R + j);
                s0 = fma(vv.x, xv[k].x, s0);
                s1 = fma(vv.y, xv[k].y, s1);
            }
            if (r2 < a.n) *reinterpret_cast<double2 *>(a.y + r2) = make_double2(s0, s1);
        } else {
            const int j = threadIdx.x;
            const int64_t r = r0 + j;
            double xv[S];
#pragma unroll
            for (int k = 0; k < S; ++k) xv[k] = __ldg(a.x + sc[k * R + j]);
            double s0 = 0.0;
#pragma unroll
            for (int k = 0; k < S; ++k) s0 = fma(sv[k * R + j], xv[k], s0);
            if (r < a.n) a.y[r] = s0;
        }
        __syncthreads();  // stage s consumed
        if (threadIdx.x == 0 && i + KS < mine) issue(i + KS, s);
    }
}

template <int R, int KS, int NT>
void run_sliced(A a, const unsigned char *sl, double alg, int sms, int per_sm, const std::vector<double> &yref) {
    const size_t sm = (size_t)R * 324 * KS;
    cudaFuncSetAttribute(tma_sliced<R, KS, NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    cudaMemset(a.y, 0, sizeof(double) * a.n);
    const float ms = best_ms([&] { tma_sliced<R, KS, NT><<<sms * per_sm, NT, sm>>>(a, sl); }, 10);
    std::vector<double> y(a.n);
    cudaMemcpy(y.data(), a.y, sizeof(double) * a.n, cudaMemcpyDeviceToHost);
    const bool ok = memcmp(y.data(), yref.data(), sizeof(double) * a.n) == 0;
    printf("{\"variant\": \"sliced_R%d_S%d_NT%d_x%d\", \"smem\": %zu, \"us\": %.1f, \"alg_GBs\": %.1f, \"bitwise\": %s, \"err\": \"%s\"}\n",
           R, KS, NT, per_sm, sm, ms * 1e3, alg / ms / 1e6, ok ? "true" : "false", cudaGetErrorString(cudaGetLastError()));
}

template <int R, int KS, int NT>
void run_tma(A a, double alg, int sms, int per_sm, const std::vector<double> &yref) {
    const size_t sm = (size_t)R * S * 12 * KS;
    cudaFuncSetAttribute(tma<R, KS, NT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    cudaMemset(a.y, 0, sizeof(double) * a.n);
    const float ms = best_ms([&] { tma<R, KS, NT><<<sms * per_sm, NT, sm>>>(a); }, 10);
    std::vector<double> y(a.n);
    cudaMemcpy(y.data(), a.y, sizeof(double) * a.n, cudaMemcpyDeviceToHost);
    const bool ok = memcmp(y.data(), yref.data(), sizeof(double) * a.n) == 0;
    printf("{\"variant\": \"tma_R%d_S%d_NT%d_x%d\", \"smem\": %zu, \"us\": %.1f, \"alg_GBs\": %.1f, \"bitwise\": %s, \"err\": \"%s\"}\n",
           R, KS, NT, per_sm, sm, ms * 1e3, alg / ms / 1e6, ok ? "true" : "false", cudaGetErrorString(cudaGetLastError()));
}

int main(int argc, char **argv) {
    const int nx = argc > 1 ? atoi(argv[1]) : 256, ny = argc > 2 ? atoi(argv[2]) : 256, nz = argc > 3 ? atoi(argv[3]) : 256;
    A a{};
    a.nx = nx;
    a.ny = ny;
    a.plane = (int64_t)nx * ny;
    a.n = a.plane * nz;
    const int64_t ncol = a.n + 2 * a.plane;
    double *x, *y, *yref_d;
    cudaMalloc(&a.val, sizeof(double) * S * a.n);
    cudaMalloc(&a.col, sizeof(int) * S * a.n);
    cudaMalloc(&x, sizeof(double) * ncol);
    cudaMalloc(&y, sizeof(double) * a.n);
    cudaMalloc(&yref_d, sizeof(double) * a.n);
    a.x = x;
    gen<<<(unsigned)((a.n + 255) / 256), 256>>>(a);
    xinit<<<(unsigned)((ncol + 255) / 256), 256>>>(x, ncol);
    const int64_t nnz = (int64_t)(3 * nx - 2) * (3 * ny - 2) * (3 * nz - 2);
    const double alg = 12.0 * nnz + 16.0 * a.n;
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    a.y = yref_d;
    ref<<<(unsigned)((a.n / 2 + 255) / 256), 256>>>(a);
    cudaDeviceSynchronize();
    std::vector<double> yref(a.n);
    cudaMemcpy(yref.data(), yref_d, sizeof(double) * a.n, cudaMemcpyDeviceToHost);
    a.y = y;
    unsigned char *sl128, *sl256;
    const int64_t nch128 = (a.n + 127) / 128, nch256 = (a.n + 255) / 256;
    cudaMalloc(&sl128, (size_t)nch128 * 128 * 324);
    unsigned char *sl64, *sl32;
    const int64_t nch64 = (a.n + 63) / 64, nch32 = (a.n + 31) / 32;
    cudaMalloc(&sl64, (size_t)nch64 * 64 * 324);
    cudaMalloc(&sl32, (size_t)nch32 * 32 * 324);
    make_sliced<64><<<(unsigned)((nch64 * 64 + 255) / 256), 256>>>(a, sl64);
    make_sliced<32><<<(unsigned)((nch32 * 32 + 255) / 256), 256>>>(a, sl32);
    cudaMalloc(&sl256, (size_t)nch256 * 256 * 324);
    make_sliced<128><<<(unsigned)((nch128 * 128 + 255) / 256), 256>>>(a, sl128);
    make_sliced<256><<<(unsigned)((nch256 * 256 + 255) / 256), 256>>>(a, sl256);
    cudaDeviceSynchronize();
    for (int rep = 0; rep < 2; ++rep) {
        const float ms = best_ms([&] { ref<<<(unsigned)((a.n / 2 + 255) / 256), 256>>>(a); }, 10);
        printf("{\"variant\": \"ref_ldg_2rows\", \"us\": %.1f, \"alg_GBs\": %.1f}\n", ms * 1e3, alg / ms / 1e6);
        run_sliced<256, 2, 256>(a, sl256, alg, sms, 1, yref);
        run_sliced<128, 2, 128>(a, sl128, alg, sms, 2, yref);
        run_sliced<64, 2, 64>(a, sl64, alg, sms, 4, yref);
        run_sliced<64, 3, 64>(a, sl64, alg, sms, 3, yref);
        run_sliced<64, 2, 64>(a, sl64, alg, sms, 5, yref);
        run_sliced<32, 4, 32>(a, sl32, alg, sms, 4, yref);
        run_sliced<32, 2, 32>(a, sl32, alg, sms, 8, yref);
    }
    return 0;
}
