// Microbenchmark: the panel's per-column "reduce P partials over all CTAs, every CTA gets
// the P sums" step (148 CTAs x 512 threads, one CTA per SM), fence-free variants.
//   0: current design: P fp64 atomics (256-byte padded), red.release counter barrier,
//      ldcg of the P sums
//   1: LL two-hop: every CTA stores its P partials as flagged 16-byte words (32-bit data
//      half + 32-bit sequence flag, twice) into slot1[p][cta]; CTA p (< P) polls the 148
//      words of entry p, sums them in CTA order and stores the sum as one flagged word into
//      slot2[p]; every CTA polls the P words of slot2
//   2: LL one hop: every CTA stores one flagged word; every CTA polls all 148 (pure
//      fence-free barrier latency)
//   3: mode 1 plus a flagged n-vector (n = 2048): each CTA stores its 14 rows, then every
//      CTA reads all n words after the sums (the GEMV operand)
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/mb_ll scripts/mb_ll.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned ld_acq(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void red_rel(unsigned *p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_ll(uint4 *p, double v, unsigned f) {
    const unsigned long long u = (unsigned long long)__double_as_longlong(v);
    asm volatile("st.relaxed.gpu.global.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"((unsigned)u), "r"(f),
                 "r"((unsigned)(u >> 32)), "r"(f)
                 : "memory");
}
__device__ __forceinline__ uint4 ld_ll(const uint4 *p) {
    uint4 r;
    asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p)
                 : "memory");
    return r;
}
__device__ __forceinline__ double poll_ll(const uint4 *p, unsigned f) {
    uint4 r = ld_ll(p);
    while (r.y != f || r.w != f) r = ld_ll(p);
    return __longlong_as_double((long long)(((unsigned long long)r.z << 32) | r.x));
}

#define P 40
#define NV 2048

__global__ void __launch_bounds__(512, 1) k_sync(int mode, int iters, unsigned *bar, double *acc, uint4 *s1,
                                                 uint4 *s2, uint4 *vec, long long *out, double *sink) {
    __shared__ double red[16];
    __shared__ double sums[P];
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = gridDim.x, b = blockIdx.x;
    unsigned epoch = 0;
    double s = 0.0;
    long long t0 = clock64();
    for (int it = 0; it < iters; it++) {
        const unsigned f = (unsigned)it + 1u;
        const double part = 1.0 + b + tid;
        if (mode == 0) {
            double *a = acc + (it & 3) * P * 32;
            if (tid < P) atomicAdd(a + tid * 32, part);
            __syncthreads();
            if (tid == 0) {
                epoch++;
                red_rel(bar, 1u);
                while (ld_acq(bar) < epoch * G) {
                }
            }
            __syncthreads();
            if (tid < P) sums[tid] = __ldcg(a + tid * 32);
            __syncthreads();
        } else if (mode == 1 || mode == 3) {
            if (mode == 3)
                for (int r = b * NV / G + tid; r < (b + 1) * NV / G; r += 512) st_ll(vec + (it & 1) * NV + r, part, f);
            if (tid < P) st_ll(s1 + tid * 256 + b, part, f);
            for (int e = b; e < P; e += G) {  // reducer of entry e
                double v = tid < G ? poll_ll(s1 + e * 256 + tid, f) : 0.0;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
                if (lane == 0 && wid < 5) red[wid] = v;
                __syncthreads();
                if (tid == 0) {
                    double t = 0.0;
                    for (int w = 0; w < 5; w++) t += red[w];
                    st_ll(s2 + e, t, f);
                }
                __syncthreads();
            }
            if (tid < P) sums[tid] = poll_ll(s2 + tid, f);
            __syncthreads();
            if (mode == 3) {
                double v = 0.0;
                for (int q = tid; q < NV; q += 512) v += poll_ll(vec + (it & 1) * NV + q, f);
                s += v;
            }
        } else if (mode == 2) {
            if (tid == 0) st_ll(s1 + (it & 1) * 256 + b, part, f);
            if (tid < G) s += poll_ll(s1 + (it & 1) * 256 + tid, f);
            __syncthreads();
        }
        if (tid < P) s += sums[tid];
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = (t1 - t0) / iters;
    if (s == -1.0) sink[0] = s;
}

int main() {
    setvbuf(stdout, NULL, _IONBF, 0);
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    unsigned *bar;
    double *acc, *sink;
    uint4 *s1, *s2, *vec;
    long long *out;
    cudaMalloc(&bar, 4096);
    cudaMalloc(&acc, 4 * P * 32 * 8);
    cudaMalloc(&s1, P * 256 * 16);
    cudaMalloc(&s2, 256 * 16);
    cudaMalloc(&vec, 2 * NV * 16);
    cudaMalloc(&sink, 8);
    cudaMalloc(&out, nsm * 8);
    const char *names[] = {"atomics + counter barrier + ldcg (P=40)", "LL two-hop reduce+bcast (P=40)",
                           "LL one-hop barrier", "LL two-hop + 2048-word LL vector"};
    for (int grid : {nsm, 74, 32}) {
        for (int mode = 0; mode < 4; mode++) {
            for (int rep = 0; rep < 2; rep++) {
                cudaMemset(bar, 0, 4096);
                cudaMemset(acc, 0, 4 * P * 32 * 8);
                cudaMemset(s1, 0, P * 256 * 16);
                cudaMemset(s2, 0, 256 * 16);
                cudaMemset(vec, 0, 2 * NV * 16);
                int iters = 2000;
                void *args[] = {&mode, &iters, &bar, &acc, &s1, &s2, &vec, &out, &sink};
                cudaEvent_t e0, e1;
                cudaEventCreate(&e0);
                cudaEventCreate(&e1);
                cudaEventRecord(e0);
                cudaLaunchCooperativeKernel((void *)k_sync, grid, 512, args, 0, 0);
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                float ms;
                cudaEventElapsedTime(&ms, e0, e1);
                long long h[256];
                cudaMemcpy(h, out, grid * 8, cudaMemcpyDeviceToHost);
                long long mx = 0;
                for (int i = 0; i < grid; i++) mx = h[i] > mx ? h[i] : mx;
                if (rep == 1)
                    printf("grid %3d  %-44s %6lld cycles/iter  %7.3f us/iter (events)\n", grid, names[mode], mx,
                           1e3 * ms / iters);
            }
        }
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
