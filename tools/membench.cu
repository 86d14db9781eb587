// membench.cu -- memory-roofline probes on the B200 (not the product):
// pure-read streams (plain / nc+no_allocate+evict_first / +L2::256B
// prefetch), a 2:1 read:write stream, and L2-resident re-reads, so the SpMV
// and vector-kernel numbers can be read against what this GPU really does.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o membench membench.cu
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdint.h>

__device__ __forceinline__ uint64_t pol_ef() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

template <int kMode>
__global__ void __launch_bounds__(256) read_kernel(const double2 *__restrict__ a, int64_t n2, double *out) {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nth = (int64_t)gridDim.x * blockDim.x;
    double s = 0.0;
    const uint64_t pol = pol_ef();
    for (int64_t i = tid; i < n2; i += 4 * nth) {
        double2 v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int64_t j = i + u * nth;
            if (j < n2) {
                if (kMode == 0) {
                    v[u] = a[j];
                } else if (kMode == 1) {
                    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;"
                        : "=d"(v[u].x), "=d"(v[u].y) : "l"(a + j), "l"(pol));
                } else {
                    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::256B.v2.f64 {%0,%1}, [%2], %3;"
                        : "=d"(v[u].x), "=d"(v[u].y) : "l"(a + j), "l"(pol));
                }
            } else {
                v[u] = make_double2(0, 0);
            }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) s += v[u].x + v[u].y;
    }
    if (s == 123.456) *out = s;
}

__global__ void __launch_bounds__(256) copy_kernel(const double2 *__restrict__ a, double2 *__restrict__ b, int64_t n2) {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nth = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = tid; i < n2; i += nth) b[i] = a[i];
}

// 2 reads : 1 write (waxpby-like)
__global__ void __launch_bounds__(256) triad_kernel(const double2 *__restrict__ a, const double2 *__restrict__ b,
                                                    double2 *__restrict__ c, int64_t n2) {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nth = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = tid; i < n2; i += nth) {
        double2 x = a[i], y = b[i];
        c[i] = make_double2(x.x + 0.5 * y.x, x.y + 0.5 * y.y);
    }
}

// CG-update-like: read x, r, p, q; write x, r (4R:2W), double2 units
__global__ void __launch_bounds__(256) upd_kernel(double2 *__restrict__ x, double2 *__restrict__ r,
                                                  const double2 *__restrict__ p, const double2 *__restrict__ q,
                                                  int64_t n2, double al) {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nth = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = tid; i < n2; i += nth) {
        double2 xa = x[i], ra = r[i];
        const double2 pa = p[i], qa = q[i];
        xa.x += al * pa.x; xa.y += al * pa.y;
        ra.x -= al * qa.x; ra.y -= al * qa.y;
        x[i] = xa;
        r[i] = ra;
    }
}

// p-update-like with the deferred x update: read r, p, x; write p, x (3R:2W)
template <int kU>
__global__ void __launch_bounds__(256) pupd_kernel(const double2 *__restrict__ r, double2 *__restrict__ p,
                                                   double2 *__restrict__ x, int64_t n2, double be, double al) {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nth = (int64_t)gridDim.x * blockDim.x;
    for (int64_t b = tid; b < n2; b += kU * nth) {
        double2 ra[kU], pa[kU], xa[kU];
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < n2) { ra[u] = r[i]; pa[u] = p[i]; xa[u] = x[i]; }
        }
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t i = b + u * nth;
            if (i < n2) {
                xa[u].x += al * pa[u].x; xa[u].y += al * pa[u].y;
                p[i] = make_double2(ra[u].x + be * pa[u].x, ra[u].y + be * pa[u].y);
                x[i] = xa[u];
            }
        }
    }
}

template <class F>
float timeit(F f, int reps) {
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
        if (ms < best) best = ms;
    }
    return best;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t big = (size_t)1 << 30;  // 1 GiB per array
    double2 *a, *b, *c;
    double *out;
    cudaMalloc(&a, big);
    cudaMalloc(&b, big);
    cudaMalloc(&c, big);
    cudaMalloc(&out, 8);
    cudaMemset(a, 0, big);
    cudaMemset(b, 0, big);
    const int64_t n2 = big / 16;
    int occ;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, read_kernel<0>, 256, 0);
    const int grid = sms * occ;
    printf("{\"sms\": %d, \"occ_read\": %d}\n", sms, occ);
    const char *names[3] = {"read_plain", "read_nc_ef", "read_nc_ef_256B"};
    for (int m = 0; m < 3; ++m) {
        float ms = timeit([&] {
            if (m == 0) read_kernel<0><<<grid, 256>>>(a, n2, out);
            if (m == 1) read_kernel<1><<<grid, 256>>>(a, n2, out);
            if (m == 2) read_kernel<2><<<grid, 256>>>(a, n2, out);
        }, 10);
        printf("{\"probe\": \"%s\", \"bytes\": %zu, \"ms\": %.4f, \"GBs\": %.1f}\n", names[m], big, ms, big / ms / 1e6);
    }
    float ms = timeit([&] { copy_kernel<<<grid, 256>>>(a, b, n2); }, 10);
    printf("{\"probe\": \"copy\", \"bytes\": %zu, \"ms\": %.4f, \"GBs\": %.1f}\n", 2 * big, ms, 2 * big / ms / 1e6);
    ms = timeit([&] { triad_kernel<<<grid, 256>>>(a, b, c, n2); }, 10);
    printf("{\"probe\": \"triad_2r1w\", \"bytes\": %zu, \"ms\": %.4f, \"GBs\": %.1f}\n", 3 * big, ms, 3 * big / ms / 1e6);
    // the 256^3 CG vectors (n = 2^24 doubles = 128 MiB each): p update with the
    // deferred x (3R:2W), one persistent wave x kU units vs a full grid
    {
        const int64_t m2 = ((int64_t)1 << 24) / 2;
        double2 *r = a, *pp = b, *xx = c;
        int o1, o4;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o1, pupd_kernel<1>, 256, 0);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o4, pupd_kernel<4>, 256, 0);
        const double bytes = 5.0 * 16 * m2;
        for (int rep = 0; rep < 2; ++rep) {
            ms = timeit([&] { pupd_kernel<1><<<(unsigned)((m2 + 255) / 256), 256>>>(r, pp, xx, m2, 0.5, 0.25); }, 10);
            printf("{\"probe\": \"pupd_3r2w_fullgrid\", \"us\": %.2f, \"GBs\": %.1f}\n", ms * 1e3, bytes / ms / 1e6);
            ms = timeit([&] { pupd_kernel<4><<<sms * o4, 256>>>(r, pp, xx, m2, 0.5, 0.25); }, 10);
            printf("{\"probe\": \"pupd_3r2w_wave_u4\", \"us\": %.2f, \"GBs\": %.1f}\n", ms * 1e3, bytes / ms / 1e6);
            ms = timeit([&] { pupd_kernel<1><<<sms * o1, 256>>>(r, pp, xx, m2, 0.5, 0.25); }, 10);
            printf("{\"probe\": \"pupd_3r2w_wave_u1\", \"us\": %.2f, \"GBs\": %.1f}\n", ms * 1e3, bytes / ms / 1e6);
            ms = timeit([&] { pupd_kernel<2><<<sms * o4 * 2, 256>>>(r, pp, xx, m2, 0.5, 0.25); }, 10);
            printf("{\"probe\": \"pupd_3r2w_2waves_u2\", \"us\": %.2f, \"GBs\": %.1f}\n", ms * 1e3, bytes / ms / 1e6);
        }
    }
    // L2-resident re-reads: 16, 32, 64 MB
    for (size_t mb : {16, 32, 64, 96}) {
        const size_t bytes = mb << 20;
        const int64_t m2 = bytes / 16;
        ms = timeit([&] { read_kernel<0><<<grid, 256>>>(a, m2, out); }, 20);
        printf("{\"probe\": \"l2_read_%zuMB\", \"bytes\": %zu, \"ms\": %.4f, \"GBs\": %.1f}\n", mb, bytes, ms, bytes / ms / 1e6);
        ms = timeit([&] { triad_kernel<<<grid, 256>>>(a, b, c, m2); }, 20);
        printf("{\"probe\": \"l2_triad_%zuMB\", \"bytes\": %zu, \"ms\": %.4f, \"GBs\": %.1f}\n", mb, 3 * bytes, ms, 3 * bytes / ms / 1e6);
    }
    // array spacing: 4 arrays of 128 MiB in one allocation, separated by
    // exactly 2^27 B vs. 2^27 B + a skew
    {
        const size_t seg = (size_t)1 << 27;
        char *base;
        cudaMalloc(&base, 4 * seg + 4 * (1 << 22));
        cudaMemset(base, 0, 4 * seg + 4 * (1 << 22));
        const int64_t m2 = seg / 16;
        for (size_t skew : {(size_t)0, (size_t)4096, (size_t)65536 + 256, (size_t)(1 << 21) + 8192}) {
            double2 *v[4];
            for (int k = 0; k < 4; ++k) v[k] = (double2 *)(base + k * (seg + skew));
            int og;
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&og, upd_kernel, 256, 0);
            ms = timeit([&] { upd_kernel<<<sms * og, 256>>>(v[0], v[1], v[2], v[3], m2, 0.5); }, 10);
            printf("{\"probe\": \"upd_4r2w_skew%zu\", \"bytes\": %zu, \"ms\": %.4f, \"GBs\": %.1f}\n", skew, 6 * seg, ms, 6 * seg / ms / 1e6);
            ms = timeit([&] { upd_kernel<<<(unsigned)((m2 + 255) / 256), 256>>>(v[0], v[1], v[2], v[3], m2, 0.5); }, 10);
            printf("{\"probe\": \"upd_4r2w_fullgrid_skew%zu\", \"bytes\": %zu, \"ms\": %.4f, \"GBs\": %.1f}\n", skew, 6 * seg, ms, 6 * seg / ms / 1e6);
        }
    }
    return 0;
}
