// Microbenchmark: dependent-latency of the FP64 / shared-memory / shuffle primitives the
// panel's column chain is built from (one warp, clock64, 1024 dependent repetitions).
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/mb_lat scripts/mb_lat.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_lat(double *out, long long *cyc, double seed) {
    __shared__ double sm[1024];
    const int lane = threadIdx.x;
    for (int i = lane; i < 1024; i += 32) sm[i] = seed * (i + 1) * 1e-9;
    __syncwarp();
    double x = seed + lane, y = 1.0 + 1e-12 * lane;
    long long t0, t1;
    const int N = 1024;
    // 0: dependent DFMA
    t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; i++) x = fma(x, y, 1e-300);
    t1 = clock64();
    if (lane == 0) cyc[0] = (t1 - t0);
    // 1: dependent DADD
    t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; i++) x = x + y;
    t1 = clock64();
    if (lane == 0) cyc[1] = (t1 - t0);
    // 2: dependent LDS (pointer chase through smem values)
    int idx = lane;
    t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; i++) idx = ((int)(sm[idx & 1023] * 1e9) + i) & 1023;
    t1 = clock64();
    if (lane == 0) cyc[2] = (t1 - t0);
    // 3: dependent double shuffle + add
    t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; i++) x += __shfl_xor_sync(0xffffffffu, x, 1 + (i & 15));
    t1 = clock64();
    if (lane == 0) cyc[3] = (t1 - t0);
    // 4: dependent sqrt
    t0 = clock64();
#pragma unroll 4
    for (int i = 0; i < N; i++) x = sqrt(x + 1.0);
    t1 = clock64();
    if (lane == 0) cyc[4] = (t1 - t0);
    // 5: dependent division
    t0 = clock64();
#pragma unroll 4
    for (int i = 0; i < N; i++) x = 1.0 / (x + 1.0);
    t1 = clock64();
    if (lane == 0) cyc[5] = (t1 - t0);
    // 6: dependent __drcp_rn
    t0 = clock64();
#pragma unroll 4
    for (int i = 0; i < N; i++) x = __drcp_rn(x + 1.0);
    t1 = clock64();
    if (lane == 0) cyc[6] = (t1 - t0);
    // 7: dependent int LDS address chain + DFMA (LDS then use)
    double acc = 0.0;
    t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; i++) acc = fma(sm[(i * 33 + lane + (int)(acc * 0.0)) & 1023], y, acc);
    t1 = clock64();
    if (lane == 0) cyc[7] = (t1 - t0);
    out[lane] = x + acc + idx;
}

int main() {
    double *out;
    long long *cyc, h[8];
    cudaMalloc(&out, 32 * 8);
    cudaMalloc(&cyc, 8 * 8);
    for (int rep = 0; rep < 2; rep++) {
        k_lat<<<1, 32>>>(out, cyc, 1.5);
        cudaMemcpy(h, cyc, 64, cudaMemcpyDeviceToHost);
    }
    const char *nm[] = {"DFMA dep", "DADD dep", "LDS dep (idx chase)", "SHFL.f64 + DADD dep", "sqrt f64 dep",
                        "div f64 dep", "__drcp_rn dep", "LDS + DFMA dep"};
    for (int i = 0; i < 8; i++) printf("%-24s %7.1f cycles\n", nm[i], h[i] / 1024.0);
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
