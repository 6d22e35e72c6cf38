// Microbenchmark: cost of the panel's per-column grid sync on this GPU (148 CTAs x 512
// threads, one CTA per SM).  Variants per iteration:
//   0: grid barrier only (warp-0 arrive/poll + named barrier release)
//   1: 20 fp64 atomics per CTA into 20 consecutive doubles, barrier, load the 20 sums
//   2: same with each accumulator in its own 256-byte block
//   3: L2 round trip only (one ldcg of a remote-written line, no barrier)
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o mb_sync scripts/mb_sync.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned ld_acq(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void red_rel(unsigned *p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ unsigned ld_rlx(const unsigned *p) {
    unsigned v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_rel(unsigned *p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// flag-array barrier: each CTA publishes its epoch in its own word; one warp polls all words
__device__ __forceinline__ void flag_barrier(unsigned *flags, unsigned epoch) {
    const int lane = threadIdx.x & 31;
    __syncwarp();
    if (lane == 0) st_rel(flags + blockIdx.x, epoch);
    while (true) {
        bool ok = true;
        for (int i = lane; i < (int)gridDim.x; i += 32) ok &= ld_rlx(flags + i) >= epoch;
        if (__all_sync(0xffffffffu, ok)) break;
    }
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    __syncwarp();
}

__global__ void __launch_bounds__(512, 1) k_sync(int mode, int iters, unsigned *bar, double *acc,
                                                 long long *out, double *sink) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    unsigned epoch = 0;
    double s = 0.0;
    long long t0 = clock64();
    for (int it = 0; it < iters; it++) {
        if (wid == 0) {
            double *a = acc + (it & 3) * 20 * 32;
            if (mode == 1 && lane < 20) atomicAdd(a + lane, 1.0);
            if (mode == 2 && lane < 20) atomicAdd(a + lane * 32, 1.0);
            if (mode >= 4) {
                double *g = acc + 4096 + (it & 3) * 8 * 32 + (blockIdx.x & 7) * 32;
                if (mode == 5 && lane < 20) atomicAdd(g + lane, 1.0);
                flag_barrier(bar + 64, it + 1);
                if (mode == 5 && lane < 20)
                    for (int q = 0; q < 8; q++) s += __ldcg(acc + 4096 + (it & 3) * 8 * 32 + q * 32 + lane);
            } else if (mode != 3) {
                __syncwarp();
                if (lane == 0) {
                    epoch++;
                    red_rel(bar, 1u);
                    while (ld_acq(bar) < epoch * gridDim.x) {
                    }
                }
                __syncwarp();
            }
            if (mode == 1 && lane < 20) s += __ldcg(a + lane);
            if (mode == 2 && lane < 20) s += __ldcg(a + lane * 32);
            if (mode == 3) s += __ldcg(acc + ((it * 37 + blockIdx.x) & 1023) * 32);
        }
        asm volatile("bar.sync 1, 512;" ::: "memory");
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = (t1 - t0) / iters;
    if (s == -1.0) sink[0] = s;
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    unsigned *bar;
    double *acc, *sink;
    long long *out;
    cudaMalloc(&bar, 4096);
    cudaMalloc(&acc, 16384 * 8);
    cudaMalloc(&sink, 8);
    cudaMalloc(&out, nsm * 8);
    cudaMemset(acc, 0, 16384 * 8);
    const char *names[] = {"barrier only", "barrier + 20 atomics (1 line)", "barrier + 20 atomics (padded)",
                           "L2 round trip (ldcg)", "flag barrier only", "flag barrier + 20 atomics (8 groups)"};
    for (int mode = 0; mode < 6; mode++) {
        for (int rep = 0; rep < 2; rep++) {
            cudaMemset(bar, 0, 4096);
            int iters = 2000;
            void *args[] = {&mode, &iters, &bar, &acc, &out, &sink};
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0);
            cudaEventCreate(&e1);
            cudaEventRecord(e0);
            cudaLaunchCooperativeKernel((void *)k_sync, nsm, 512, args, 0, 0);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            long long h[256];
            cudaMemcpy(h, out, nsm * 8, cudaMemcpyDeviceToHost);
            long long mx = 0;
            for (int i = 0; i < nsm; i++) mx = h[i] > mx ? h[i] : mx;
            if (rep == 1)
                printf("%-34s %8lld cycles/iter (max over CTAs)  %7.3f us/iter (events)\n", names[mode], mx,
                       1e3 * ms / iters);
        }
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
