// Microbenchmark: how many warps / which warp tile the FP64 DMMA pipe needs to run at its peak
// when the fragments come from shared memory (the update GEMMs' inner loop), no global traffic.
//   reg<W, ACC>:  register-resident DMMA, W warps per SM, ACC independent accumulators per warp
//   smem<MI, NI, NW, CPS>: an (8 MI x 8 NI) warp tile fed by LDS from k-major 64 x 68 tiles
//                          (stride 68: conflict free), NW warps per CTA, CPS CTAs per SM
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/mb_gemm scripts/mb_gemm.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void dmma(double &d0, double &d1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(d0), "+d"(d1)
                 : "d"(a), "d"(b));
}

template <int ACC>
__global__ void k_reg(double *out, int iters) {
    double d[ACC][2];
    for (int i = 0; i < ACC; i++) d[i][0] = d[i][1] = 0.0;
    double a = 1.0 + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int i = 0; i < ACC; i++) dmma(d[i][0], d[i][1], a, b);
    }
    double s = 0.0;
    for (int i = 0; i < ACC; i++) s += d[i][0] + d[i][1];
    if (s == 1234.5) out[threadIdx.x] = s;
}

#define SK 68
template <int MI, int NI, int NW>
__global__ void __launch_bounds__(NW * 32) k_smem(double *out, int iters) {
    extern __shared__ double sm[];
    double(*As)[SK] = reinterpret_cast<double(*)[SK]>(sm);
    double(*Bs)[SK] = reinterpret_cast<double(*)[SK]>(sm + 64 * SK);
    for (int i = threadIdx.x; i < 2 * 64 * SK; i += blockDim.x) sm[i] = 1.0 + 1e-12 * i;
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, lr = lane >> 2, lc = lane & 3;
    // warps tile the 64 x 64 block: (64 / (8 MI)) x (64 / (8 NI)) warp positions (wrapped)
    constexpr int WX = 64 / (8 * MI), WY = 64 / (8 * NI);
    const int wx = warp % WX, wy = (warp / WX) % WY;
    double acc[MI][NI][2];
#pragma unroll
    for (int i = 0; i < MI; i++)
#pragma unroll
        for (int j = 0; j < NI; j++) acc[i][j][0] = acc[i][j][1] = 0.0;
    for (int it = 0; it < iters; it++) {
#pragma unroll 4
        for (int k0 = 0; k0 < 64; k0 += 4) {
            double a[MI], b[NI];
#pragma unroll
            for (int i = 0; i < MI; i++) a[i] = As[k0 + lc][wx * 8 * MI + i * 8 + lr];
#pragma unroll
            for (int j = 0; j < NI; j++) b[j] = Bs[k0 + lc][wy * 8 * NI + j * 8 + lr];
#pragma unroll
            for (int i = 0; i < MI; i++)
#pragma unroll
                for (int j = 0; j < NI; j++) dmma(acc[i][j][0], acc[i][j][1], a[i], b[j]);
        }
    }
    double s = 0.0;
#pragma unroll
    for (int i = 0; i < MI; i++)
#pragma unroll
        for (int j = 0; j < NI; j++) s += acc[i][j][0] + acc[i][j][1];
    if (s == 1234.5) out[threadIdx.x] = s;
}

static cudaEvent_t e0, e1;
static int nsm;
static double *out;

template <int ACC>
void run_reg(int wps) {
    const int iters = 4000;
    const int blocks = nsm, threads = wps * 32;
    float best = 1e30f;
    for (int rep = 0; rep < 3; rep++) {
        cudaEventRecord(e0);
        k_reg<ACC><<<blocks, threads>>>(out, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    const double fl = (double)blocks * wps * iters * ACC * 512.0;
    printf("reg   warps/SM=%2d acc/warp=%2d : %6.1f TFLOP/s\n", wps, ACC, fl / best / 1e9);
}

template <int MI, int NI, int NW>
void run_smem(int cps) {
    const int iters = 200;
    const size_t smem = 2 * 64 * SK * 8;
    cudaFuncSetAttribute(k_smem<MI, NI, NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_smem<MI, NI, NW>, NW * 32, smem);
    const int c = cps < occ ? cps : occ;
    const int blocks = nsm * c;
    float best = 1e30f;
    for (int rep = 0; rep < 3; rep++) {
        cudaEventRecord(e0);
        k_smem<MI, NI, NW><<<blocks, NW * 32, smem>>>(out, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, k_smem<MI, NI, NW>);
    const double fl = (double)blocks * NW * iters * 16.0 * MI * NI * 512.0;
    printf("smem  warp tile %2dx%2d  warps/CTA=%2d CTAs/SM=%d (occ %d, %3d regs) : %6.1f TFLOP/s  (LDS/DMMA %.2f)\n",
           8 * MI, 8 * NI, NW, c, occ, fa.numRegs, fl / best / 1e9, (double)(MI + NI) / (MI * NI));
}

int main() {
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    cudaMalloc(&out, 1 << 16);
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    run_reg<8>(32);  // warm-up
    for (int w : {4, 8, 16, 32}) {
        run_reg<4>(w);
        run_reg<8>(w);
        run_reg<16>(w);
    }
    run_smem<2, 4, 8>(1);
    run_smem<2, 4, 8>(2);
    run_smem<2, 4, 16>(1);
    run_smem<4, 4, 8>(1);
    run_smem<4, 4, 8>(2);
    run_smem<4, 4, 16>(1);
    run_smem<4, 8, 4>(1);
    run_smem<4, 8, 8>(1);
    run_smem<4, 8, 8>(2);


    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
