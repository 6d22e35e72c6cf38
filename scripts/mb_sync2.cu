// Microbenchmark: grid-barrier variants for the panel kernel (148 CTAs x 512 threads,
// cooperative launch), cycles per barrier (max over CTAs).  Each iteration: bar.sync,
// thread 0 arrives/polls, bar.sync.
//   0: one counter, red.release + ld.acquire poll (the panel kernel's barrier)
//   1: one counter, fence.acq_rel + red.relaxed, poll ld.relaxed, fence.acq_rel after
//   2: 8 striped counters (CTA i -> counter i % 8), lanes 0..7 poll with ld.acquire
//   3: 8 striped counters, red.release; lane q polls counter q with ld.relaxed; one fence after
//   4: variant 0 with the poll done by a spinning warp with nanosleep(32)
//   5: one counter, atom.add.release (returning) instead of red
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/mb_sync2 scripts/mb_sync2.cu
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned ld_acq(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned ld_rlx(const unsigned *p) {
    unsigned v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void red_rel(unsigned *p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_rlx(unsigned *p, unsigned v) {
    asm volatile("red.relaxed.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned atom_rel(unsigned *p, unsigned v) {
    unsigned r;
    asm volatile("atom.release.gpu.global.add.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "r"(v) : "memory");
    return r;
}
__global__ void __launch_bounds__(512, 1) k(int mode, int iters, unsigned *bar, long long *out) {
    const int tid = threadIdx.x, lane = tid & 31;
    const unsigned P = gridDim.x;
    long long t0 = clock64();
    for (int it = 1; it <= iters; it++) {
        __syncthreads();
        if (mode == 0 || mode == 4 || mode == 5) {
            if (tid == 0) {
                if (mode == 5) atom_rel(bar, 1u);
                else red_rel(bar, 1u);
                while (ld_acq(bar) < it * P) {
                    if (mode == 4) __nanosleep(32);
                }
            }
        } else if (mode == 1) {
            if (tid == 0) {
                asm volatile("fence.acq_rel.gpu;" ::: "memory");
                red_rlx(bar, 1u);
                while (ld_rlx(bar) < it * P) {
                }
                asm volatile("fence.acq_rel.gpu;" ::: "memory");
            }
        } else if (mode == 2 || mode == 3) {
            if (tid < 32) {
                unsigned *ctr = bar + 64 * (blockIdx.x & 7);
                if (lane == 0) {
                    red_rel(ctr, 1u);
                }
                const unsigned cnt = (P - lane + 7) / 8;  // CTAs with blockIdx % 8 == lane
                while (true) {
                    bool ok = true;
                    if (lane < 8) ok = (mode == 2 ? ld_acq(bar + 64 * lane) : ld_rlx(bar + 64 * lane)) >= it * cnt;
                    if (__all_sync(0xffffffffu, ok)) break;
                }
                if (mode == 3) asm volatile("fence.acq_rel.gpu;" ::: "memory");
            }
        }
        __syncthreads();
    }
    long long t1 = clock64();
    if (tid == 0) out[blockIdx.x] = (t1 - t0) / iters;
}
int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    unsigned *bar;
    long long *out;
    cudaMalloc(&bar, 65536);
    cudaMalloc(&out, 256 * 8);
    const char *names[] = {"counter red.release / ld.acquire", "counter fence+red.relaxed / ld.relaxed+fence",
                           "8 striped counters, ld.acquire", "8 striped counters, ld.relaxed + fence",
                           "counter, poll with nanosleep(32)", "counter atom.release (returning)"};
    int grids[] = {148, 74, 32};
    for (int gi = 0; gi < 3; gi++)
        for (int mode = 0; mode < 6; mode++) {
            int grid = grids[gi] < nsm ? grids[gi] : nsm;
            long long mx = 0;
            float ms = 0;
            for (int rep = 0; rep < 2; rep++) {
                cudaMemset(bar, 0, 65536);
                int iters = 4000;
                void *args[] = {&mode, &iters, &bar, &out};
                cudaEvent_t e0, e1;
                cudaEventCreate(&e0);
                cudaEventCreate(&e1);
                cudaEventRecord(e0);
                cudaLaunchCooperativeKernel((void *)k, grid, 512, args, 0, 0);
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                cudaEventElapsedTime(&ms, e0, e1);
                long long h[256];
                cudaMemcpy(h, out, grid * 8, cudaMemcpyDeviceToHost);
                mx = 0;
                for (int i = 0; i < grid; i++) mx = h[i] > mx ? h[i] : mx;
                ms = 1e3f * ms / iters;
            }
            printf("grid %3d  %-46s %6lld cycles  %6.3f us/barrier\n", grid, names[mode], mx, ms);
        }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
