// ringbench.cu -- probe (not the product): cost of the p update's vector
// streams at 256^3 (n = 16.7M doubles per vector) for the deferred x update
// applied every iteration (3R:2W in place: r, p, x -> p, x) against an
// m-iteration deferral over a ring of p buffers: (m - 1) iterations of 2R:1W
// (r, p_k -> p_k+1) and one flush iteration (r, p_k, x and the m - 1 older
// p's -> p_k+1, x).  An 800 MB buffer is swept between launches so every
// launch starts with a cold L2 (the SpMV streams 5.4 GB between p updates).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ringbench ringbench.cu
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdint.h>
#include <vector>

constexpr int kB = 256;

// in place: p = r + b p, x += a p  (current product pattern)
__global__ void __launch_bounds__(kB) upd_inplace(const double2 *__restrict__ r, double2 *__restrict__ p,
                                                  double2 *__restrict__ x, int64_t n2, double a, double b) {
    const int64_t tid = (int64_t)blockIdx.x * kB + threadIdx.x, nth = (int64_t)gridDim.x * kB;
    for (int64_t i = tid; i < n2; i += nth) {
        const double2 rv = r[i], pv = p[i];
        double2 xv = x[i];
        xv.x = fma(a, pv.x, xv.x);
        xv.y = fma(a, pv.y, xv.y);
        x[i] = xv;
        p[i] = make_double2(fma(b, pv.x, rv.x), fma(b, pv.y, rv.y));
    }
}

// ring, no flush: q = r + b p
__global__ void __launch_bounds__(kB) upd_ring(const double2 *__restrict__ r, const double2 *__restrict__ p,
                                               double2 *__restrict__ q, int64_t n2, double b) {
    const int64_t tid = (int64_t)blockIdx.x * kB + threadIdx.x, nth = (int64_t)gridDim.x * kB;
    for (int64_t i = tid; i < n2; i += nth) {
        const double2 rv = r[i], pv = p[i];
        q[i] = make_double2(fma(b, pv.x, rv.x), fma(b, pv.y, rv.y));
    }
}

struct Old {
    const double2 *p[16];
};

// ring flush: q = r + b p; x += sum_j a_j old_j (j ascending, old_{m-1} = p)
template <int kM>
__global__ void __launch_bounds__(kB) upd_flush(const double2 *__restrict__ r, const double2 *__restrict__ p,
                                                double2 *__restrict__ q, double2 *__restrict__ x, Old o,
                                                int64_t n2, double a, double b) {
    const int64_t tid = (int64_t)blockIdx.x * kB + threadIdx.x, nth = (int64_t)gridDim.x * kB;
    for (int64_t i = tid; i < n2; i += nth) {
        const double2 rv = r[i], pv = p[i];
        double2 xv = x[i];
        double2 ov[kM > 1 ? kM - 1 : 1];
#pragma unroll
        for (int j = 0; j < kM - 1; ++j) ov[j] = __ldcs(o.p[j] + i);
#pragma unroll
        for (int j = 0; j < kM - 1; ++j) {
            xv.x = fma(a, ov[j].x, xv.x);
            xv.y = fma(a, ov[j].y, xv.y);
        }
        xv.x = fma(a, pv.x, xv.x);
        xv.y = fma(a, pv.y, xv.y);
        x[i] = xv;
        q[i] = make_double2(fma(b, pv.x, rv.x), fma(b, pv.y, rv.y));
    }
}

__global__ void sweep(double2 *f, int64_t n2) {
    const int64_t tid = (int64_t)blockIdx.x * kB + threadIdx.x, nth = (int64_t)gridDim.x * kB;
    for (int64_t i = tid; i < n2; i += nth) f[i].x += 1.0;
}

int main(int argc, char **argv) {
    const int64_t n = (int64_t)256 * 256 * 256, n2 = n / 2;
    const int R = 17;
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    std::vector<double2 *> ring(R);
    for (auto &b : ring) cudaMalloc(&b, n * 8), cudaMemset(b, 0, n * 8);
    double2 *r, *x, *fl;
    cudaMalloc(&r, n * 8);
    cudaMalloc(&x, n * 8);
    const int64_t fn2 = (int64_t)800 << 20 >> 4;
    cudaMalloc(&fl, fn2 * 16);
    cudaMemset(r, 0, n * 8);
    cudaMemset(x, 0, n * 8);
    cudaMemset(fl, 0, fn2 * 16);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int grid = nsm * 8;  // 8 x 256 threads per SM
    auto timeit = [&](auto fn) {
        float best = 1e9, tot = 0;
        const int reps = 10;
        for (int it = 0; it < reps + 2; ++it) {
            sweep<<<nsm * 8, kB>>>(fl, fn2);
            cudaEventRecord(e0);
            fn();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (it >= 2) {
                tot += ms;
                if (ms < best) best = ms;
            }
        }
        return 1e3 * tot / reps;
    };
    const double t_in = timeit([&] { upd_inplace<<<grid, kB>>>(r, ring[0], x, n2, 0.5, 0.25); });
    const double t_ring = timeit([&] { upd_ring<<<grid, kB>>>(r, ring[0], ring[1], n2, 0.25); });
    printf("in place 3R:2W  %8.2f us  (%.0f GB/s on 40n)\n", t_in, 40.0 * n / t_in / 1e3);
    printf("ring     2R:1W  %8.2f us  (%.0f GB/s on 24n)\n", t_ring, 24.0 * n / t_ring / 1e3);
    auto flush = [&](auto kern, int m) {
        Old o{};
        for (int j = 0; j < m - 1; ++j) o.p[j] = ring[2 + j];
        const double t = timeit([&] { kern<<<grid, kB>>>(r, ring[0], ring[1], x, o, n2, 0.5, 0.25); });
        const double avg = ((m - 1) * t_ring + t) / m;
        printf("flush m=%2d      %8.2f us  (%.0f GB/s on %dn)  per-iteration average %.2f us (saves %.2f)\n", m,
               t, (40.0 + 8 * (m - 1)) * n / t / 1e3, 40 + 8 * (m - 1), avg, t_in - avg);
    };
    flush(upd_flush<2>, 2);
    flush(upd_flush<4>, 4);
    flush(upd_flush<6>, 6);
    flush(upd_flush<8>, 8);
    flush(upd_flush<12>, 12);
    flush(upd_flush<16>, 16);
    cudaError_t e = cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(e));
    return 0;
}
