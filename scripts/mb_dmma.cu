// Microbenchmark: FP64 peak of this B200 -- register-resident DMMA m8n8k4 (tensor pipe) and
// DFMA (CUDA cores) loops, all SMs, CUDA events.  The roofline denominator of the update GEMMs.
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/mb_dmma scripts/mb_dmma.cu
#include <cstdio>
#include <cuda_runtime.h>
__global__ void __launch_bounds__(256) k_dmma(double *out, int iters) {
    double d[8][2];
    for (int i = 0; i < 8; i++) d[i][0] = d[i][1] = 0.0;
    double a = 1.0 + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int i = 0; i < 8; i++)
            asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                         : "+d"(d[i][0]), "+d"(d[i][1])
                         : "d"(a), "d"(b));
    }
    double s = 0.0;
    for (int i = 0; i < 8; i++) s += d[i][0] + d[i][1];
    if (s == 1234.5) out[threadIdx.x] = s;
}
__global__ void __launch_bounds__(256) k_dfma(double *out, int iters) {
    double x[8];
    for (int i = 0; i < 8; i++) x[i] = threadIdx.x * 1e-9 + i;
    const double a = 0.999999, b = 1e-7;
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int i = 0; i < 8; i++) x[i] = fma(x[i], a, b);
    }
    double s = 0.0;
    for (int i = 0; i < 8; i++) s += x[i];
    if (s == 1234.5) out[threadIdx.x] = s;
}
int main(int argc, char **argv) {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    double *out;
    cudaMalloc(&out, 4096);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int iters = 20000, blocks = nsm * 4;
    const double fl_dmma = (double)blocks * 8 * iters * 8 * 512;  // warps * DMMA * flop
    const double fl_dfma = (double)blocks * 256 * iters * 8 * 2;
    double burst = 0.0, dfma = 0.0;
    for (int rep = 0; rep < 3; rep++) {  // burst: best of 3 single launches (~10 ms each)
        float ms, ms2;
        cudaEventRecord(e0);
        k_dmma<<<blocks, 256>>>(out, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        cudaEventRecord(e0);
        k_dfma<<<blocks, 256>>>(out, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms2, e0, e1);
        if (fl_dmma / ms / 1e9 > burst) burst = fl_dmma / ms / 1e9;
        if (fl_dfma / ms2 / 1e9 > dfma) dfma = fl_dfma / ms2 / 1e9;
    }
    // sustained: back-to-back launches for ~4 s (the update GEMMs run inside seconds-long steps)
    int nl = 0;
    float tot = 0.f;
    cudaEventRecord(e0);
    for (; nl < 100000; nl++) {
        k_dmma<<<blocks, 256>>>(out, iters);
        if (nl % 50 == 49) {
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&tot, e0, e1);
            if (tot > 4000.f) {
                nl++;
                break;
            }
        }
    }
    const double sustained = fl_dmma * nl / tot / 1e9;
    printf("DMMA m8n8k4: %.1f TFLOP/s burst, %.1f TFLOP/s sustained (%d launches, %.1f s)   DFMA: %.1f TFLOP/s   "
           "(%d SMs, %d blocks x 256)\n", burst, sustained, nl, tot / 1e3, dfma, nsm, blocks);
    if (argc > 1) {
        FILE *f = fopen(argv[1], "w");
        if (f) {
            fprintf(f, "{\"dmma_tflops\": %.2f, \"dmma_tflops_sustained\": %.2f, \"dfma_tflops\": %.2f, \"sms\": %d, "
                       "\"how\": \"scripts/mb_dmma.cu: register-resident mma.sync m8n8k4 f64 (SASS DMMA.8x8x4), %d blocks x 8 warps "
                       "x 8 independent accumulators; burst = best of 3 ~10 ms launches, sustained = back-to-back launches "
                       "for ~4 s; DFMA = fma.rn.f64 chains\"}\n", burst, sustained, dfma, nsm, blocks);
            fclose(f);
        }
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
