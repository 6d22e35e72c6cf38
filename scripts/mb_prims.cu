// Microbenchmark: latency of the panel kernel's CTA-level primitives (one CTA of 512 threads,
// or 148 CTAs), cycles per iteration measured with clock64 by thread 0.  nvcc -arch=sm_100a.
#include <cstdio>
#include <cuda_runtime.h>
#define PT 512
__device__ __forceinline__ double g8(double v) {
    v += __shfl_xor_sync(0xffffffffu, v, 4);
    v += __shfl_xor_sync(0xffffffffu, v, 2);
    v += __shfl_xor_sync(0xffffffffu, v, 1);
    return v;
}
template <int MODE>
__global__ void __launch_bounds__(PT, 1) k(double *out, long long *cyc, int iters, int J, int R) {
    __shared__ double X[64 * 65];
    __shared__ double z[64];
    __shared__ double o[512];
    const int tid = threadIdx.x, slot = tid >> 3, g = tid & 7, wid = tid >> 5;
    for (int i = tid; i < 64 * 65; i += PT) X[i] = 1e-3 * (i % 17);
    if (tid < 64) z[tid] = 0.5;
    __syncthreads();
    double acc = 0.0;
    long long t0 = clock64();
    for (int it = 0; it < iters; it++) {
        if (MODE == 0) {  // bar.sync only
            __syncthreads();
        } else if (MODE == 1) {  // 8-lane rowdot (unrolled, predicated) + bar
            if (4 * wid < R) {
                double s0 = 0, s1 = 0;
                if (slot < R) {
                    const double *x = X + slot * 65;
#pragma unroll
                    for (int u = 0; u < 8; u += 2) {
                        int a = g + 8 * u, b = a + 8;
                        if (a < J) s0 += x[a] * z[a];
                        if (b < J) s1 += x[b] * z[b];
                    }
                }
                double s = g8(s0 + s1);
                if (g == 0 && slot < R) o[slot] = s;
            }
            __syncthreads();
        } else if (MODE == 2) {  // one LDS -> DFMA -> STS dependent chain + bar
            o[tid] = o[tid] * 1.0000001 + z[tid & 63];
            __syncthreads();
        } else if (MODE == 3) {  // shuffle x3 (double) + bar
            double v = o[tid];
            v = g8(v);
            o[tid] = v;
            __syncthreads();
        } else if (MODE == 4) {  // rowdot w/o shuffle
            if (4 * wid < R) {
                double s0 = 0, s1 = 0;
                if (slot < R) {
                    const double *x = X + slot * 65;
#pragma unroll
                    for (int u = 0; u < 8; u += 2) {
                        int a = g + 8 * u, b = a + 8;
                        if (a < J) s0 += x[a] * z[a];
                        if (b < J) s1 += x[b] * z[b];
                    }
                }
                if (slot < R) o[tid] = s0 + s1;
            }
            __syncthreads();
        } else if (MODE == 5) {  // warp-only (no bar) rowdot+shuffle in warp 0
            if (wid == 0) {
                double s0 = 0, s1 = 0;
                const double *x = X + slot * 65;
#pragma unroll
                for (int u = 0; u < 8; u += 2) {
                    int a = g + 8 * u, b = a + 8;
                    if (a < J) s0 += x[a] * z[a];
                    if (b < J) s1 += x[b] * z[b];
                }
                double s = g8(s0 + s1);
                if (g == 0) o[slot] = s;
                __syncwarp();
            }
        } else if (MODE == 6) {  // DLARFG scalars: sqrt, two divisions (warp 0, dependent chain)
            if (wid == 0) {
                const double al = o[tid] + 1.5, nr = z[tid & 63] + 2.0;
                const double be = -copysign(sqrt(al * al + nr), al);
                const double ta = (be - al) / be, sc = 1.0 / (al - be);
                o[tid] = ta * sc * 1e-300;
                __syncwarp();
            }
        } else if (MODE == 7) {  // L2 round trip: ldcg of a global written by nobody
            if (tid == 0) o[0] += __ldcg(out + 1000000 + (it & 7) * 32);
            __syncthreads();
        }
        acc += o[tid & 511];
    }
    long long t1 = clock64();
    if (tid == 0) cyc[blockIdx.x] = (t1 - t0) / iters;
    out[blockIdx.x * PT + tid] = acc;
}

template <int M>
void run(const char *name, int grid, int J, int R) {
    double *out;
    long long *cyc, h[148];
    cudaMalloc(&out, sizeof(double) * (148 * PT + 1000000 + 1024));
    cudaMemset(out, 0, sizeof(double) * (148 * PT + 1000000 + 1024));
    cudaMalloc(&cyc, sizeof(long long) * 148);
    const int iters = 2000;
    k<M><<<grid, PT>>>(out, cyc, iters, J, R);
    k<M><<<grid, PT>>>(out, cyc, iters, J, R);
    cudaDeviceSynchronize();
    cudaMemcpy(h, cyc, sizeof(long long) * grid, cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < grid; i++) mx = h[i] > mx ? h[i] : mx;
    printf("%-44s grid=%3d J=%2d R=%3d  %6lld cycles/iter (max over CTAs)\n", name, grid, J, R, mx);
    cudaFree(out);
    cudaFree(cyc);
}
int main() {
    run<0>("bar.sync (512 thr)", 1, 32, 14);
    run<0>("bar.sync (512 thr)", 148, 32, 14);
    run<2>("LDS->DFMA->STS + bar", 1, 32, 14);
    run<3>("3x double shuffle + bar", 1, 32, 14);
    run<4>("rowdot (no shuffle) + bar", 1, 32, 14);
    run<1>("rowdot + g8 shuffle + bar", 1, 32, 14);
    run<1>("rowdot + g8 shuffle + bar", 1, 64, 14);
    run<1>("rowdot + g8 shuffle + bar", 1, 64, 64);
    run<1>("rowdot + g8 shuffle + bar", 148, 32, 14);
    run<5>("rowdot + g8 shuffle, warp 0 only", 1, 32, 14);
    run<6>("DLARFG scalars (sqrt + 2 div), warp 0", 1, 32, 14);
    run<7>("ldcg L2 round trip + bar", 1, 32, 14);
    run<7>("ldcg L2 round trip + bar", 148, 32, 14);
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
