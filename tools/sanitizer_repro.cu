// sanitizer_repro.cu -- minimal reproducers for the two compute-sanitizer
// reports left open in round 1, independent of the
// library: ONE kernel with the library's reduction pattern (grid-stride dot,
// warp shuffle -> shared memory -> __syncthreads -> warp 0, then the
// last-block-done grid sum), launched four ways:
//
//   plain   an ordinary launch
//   pdl     after another kernel, with programmatic dependent launch and
//           griddepcontrol.wait / launch_dependents in the kernel (as the
//           library's CG / Fig. 12 kernels do)
//   graph   inside a captured CUDA graph (no conditional node)
//   while   inside the body of a conditional WHILE node (3 iterations)
//
// and two kernel bodies: kTail = 0 (one grid-stride loop; lanes leave it at
// different trips) and kTail = 1 (the tri_dot_kernel shape: full trips, then a
// fixed-count ragged tail so no lane leaves early).  The result is checked
// against a host sum, so the kernel is demonstrably correct whatever the tool
// prints.  Build and run (tools/sanitize.sh runs it under each tool):
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o sanitizer_repro sanitizer_repro.cu
//   compute-sanitizer --tool synccheck ./sanitizer_repro pdl 1
#include <cuda_runtime.h>
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

constexpr int kBlock = 256, kWarps = kBlock / 32, kU = 4;

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

__device__ __forceinline__ double block_sum(double v, double *sh) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    __syncwarp();
    v = warp_sum(v);
    if (lane == 0) sh[warp] = v;
    __syncwarp();
    __syncthreads();
    if (warp == 0) {
        v = lane < kWarps ? sh[lane] : 0.0;
        v = warp_sum(v);
    }
    return v;
}

template <int kTail, bool kPdl>
__global__ void __launch_bounds__(kBlock) dot_kernel(long n, const double *x, const double *y, double *parts,
                                                     unsigned *counter, double *out) {
    __shared__ double sh[32];
    __shared__ int is_last;
    if (kPdl) {
        asm volatile("griddepcontrol.wait;" ::: "memory");
        asm volatile("griddepcontrol.launch_dependents;");
    }
    const long nth = (long)gridDim.x * kBlock;
    long b0 = (long)blockIdx.x * kBlock + threadIdx.x;
    double acc = 0.0;
    if (kTail) {
        const long full = n / (kU * nth) * (kU * nth);
        for (; b0 < full; b0 += kU * nth) {
            double xv[kU], yv[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                xv[u] = x[b0 + u * nth];
                yv[u] = y[b0 + u * nth];
            }
#pragma unroll
            for (int u = 0; u < kU; ++u) acc = fma(xv[u], yv[u], acc);
        }
#pragma unroll
        for (int t = 0; t < kU; ++t) {
            const long i = b0 + t * nth;
            if (i < n) acc = fma(x[i], y[i], acc);
        }
    } else {
        for (long i = b0; i < n; i += nth) acc = fma(x[i], y[i], acc);
    }
    acc = block_sum(acc, sh);
    if (threadIdx.x == 0) {
        parts[blockIdx.x] = acc;
        __threadfence();
        is_last = atomicAdd(counter, 1u) == gridDim.x - 1;
    }
    __syncwarp();
    __syncthreads();
    if (!is_last) return;
    __threadfence();
    double s = 0.0;
    for (unsigned i = threadIdx.x; i < gridDim.x; i += kBlock) s += __ldcg(parts + i);
    __syncthreads();
    s = block_sum(s, sh);
    if (threadIdx.x == 0) {
        *counter = 0u;
        *out += s;  // accumulate over the launches (checked on the host)
    }
}

__global__ void touch_kernel(double *p) {
    if (threadIdx.x == 0 && blockIdx.x == 0) p[0] += 0.0;
    asm volatile("griddepcontrol.launch_dependents;");
}

__global__ void cond_kernel(cudaGraphConditionalHandle h, int *left) {
    const int l = --*left;
    cudaGraphSetConditional(h, l > 0 ? 1u : 0u);
}

#define CK(x)                                                                            \
    do {                                                                                 \
        cudaError_t e = (x);                                                             \
        if (e != cudaSuccess) {                                                          \
            fprintf(stderr, "%s: %s (line %d)\n", #x, cudaGetErrorString(e), __LINE__); \
            exit(2);                                                                     \
        }                                                                                \
    } while (0)

template <int kTail>
int run(const char *mode) {
    const long n = 1000003;  // ragged: not a multiple of any trip
    const int grid = 148 * 4;
    double *x, *y, *parts, *out, *scratch;
    unsigned *counter;
    int *left;
    CK(cudaMalloc(&x, n * sizeof(double)));
    CK(cudaMalloc(&y, n * sizeof(double)));
    CK(cudaMalloc(&parts, grid * sizeof(double)));
    CK(cudaMalloc(&out, sizeof(double)));
    CK(cudaMalloc(&scratch, sizeof(double)));
    CK(cudaMalloc(&counter, sizeof(unsigned)));
    CK(cudaMalloc(&left, sizeof(int)));
    double *hx = (double *)malloc(n * sizeof(double)), *hy = (double *)malloc(n * sizeof(double));
    double ref = 0.0;
    for (long i = 0; i < n; ++i) {  // integer-valued: every order gives the exact sum
        hx[i] = (double)(i % 7);
        hy[i] = (double)(i % 5);
        ref += hx[i] * hy[i];
    }
    CK(cudaMemcpy(x, hx, n * sizeof(double), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(y, hy, n * sizeof(double), cudaMemcpyHostToDevice));
    CK(cudaMemset(out, 0, sizeof(double)));
    CK(cudaMemset(scratch, 0, sizeof(double)));
    CK(cudaMemset(counter, 0, sizeof(unsigned)));
    cudaStream_t st;
    CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    int launches = 1;
    if (!strcmp(mode, "plain")) {
        dot_kernel<kTail, false><<<grid, kBlock, 0, st>>>(n, x, y, parts, counter, out);
    } else if (!strcmp(mode, "pdl")) {
        touch_kernel<<<grid, kBlock, 0, st>>>(scratch);
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(grid);
        cfg.blockDim = dim3(kBlock);
        cfg.stream = st;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        CK(cudaLaunchKernelEx(&cfg, dot_kernel<kTail, true>, n, (const double *)x, (const double *)y, parts,
                              counter, out));
    } else if (!strcmp(mode, "graph")) {
        cudaGraph_t g;
        cudaGraphExec_t ge;
        CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
        dot_kernel<kTail, false><<<grid, kBlock, 0, st>>>(n, x, y, parts, counter, out);
        CK(cudaStreamEndCapture(st, &g));
        CK(cudaGraphInstantiate(&ge, g, 0));
        CK(cudaGraphLaunch(ge, st));
    } else if (!strcmp(mode, "while")) {
        launches = 3;
        const int three = 3;
        CK(cudaMemcpy(left, &three, sizeof(int), cudaMemcpyHostToDevice));
        cudaGraph_t g, body;
        cudaGraphExec_t ge;
        CK(cudaGraphCreate(&g, 0));
        cudaGraphConditionalHandle h;
        CK(cudaGraphConditionalHandleCreate(&h, g, 1u, cudaGraphCondAssignDefault));
        cudaGraphNodeParams cp{};
        cp.type = cudaGraphNodeTypeConditional;
        cp.conditional.handle = h;
        cp.conditional.type = cudaGraphCondTypeWhile;
        cp.conditional.size = 1;
        cudaGraphNode_t wn;
        CK(cudaGraphAddNode(&wn, g, nullptr, 0, &cp));
        body = cp.conditional.phGraph_out[0];
        CK(cudaStreamBeginCaptureToGraph(st, body, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal));
        dot_kernel<kTail, false><<<grid, kBlock, 0, st>>>(n, x, y, parts, counter, out);
        cond_kernel<<<1, 1, 0, st>>>(h, left);
        CK(cudaStreamEndCapture(st, &body));
        CK(cudaGraphInstantiate(&ge, g, 0));
        CK(cudaGraphLaunch(ge, st));
    } else {
        fprintf(stderr, "mode: plain | pdl | graph | while\n");
        return 2;
    }
    CK(cudaStreamSynchronize(st));
    double got = 0.0;
    CK(cudaMemcpy(&got, out, sizeof(double), cudaMemcpyDeviceToHost));
    const bool ok = got == launches * ref;
    printf("mode=%s tail=%d launches=%d sum=%.1f expected=%.1f %s\n", mode, kTail, launches, got,
           launches * ref, ok ? "OK" : "MISMATCH");
    return ok ? 0 : 1;
}

int main(int argc, char **argv) {
    const char *mode = argc > 1 ? argv[1] : "plain";
    const int tail = argc > 2 ? atoi(argv[2]) : 1;
    return tail ? run<1>(mode) : run<0>(mode);
}
