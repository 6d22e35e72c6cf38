// Microbenchmark: is the per-SM streaming rate of the panel GEMV a property of the SM?  One CTA
// per SM (512 threads, the wide panel's shape) streams its own equal row slab of every column of a
// column-major 16384 x 16384 matrix (the GEMV partition); each CTA records %smid and its
// globaltimer span.  Repeated launches: the correlation of the per-SM spans between launches says
// whether a static per-SM row weighting could balance the panel's column barrier.
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/mb_smbw scripts/mb_smbw.cu
#include <cmath>
#include <cstdlib>
#include <cstdio>
#include <cuda_runtime.h>
#include <vector>

__global__ void __launch_bounds__(512, 1) k_slab(const double *__restrict__ A, int n, int64_t ld, int R,
                                                 const double *__restrict__ x, double *y, unsigned long long *rec,
                                                 int rb = 0, int cb = 0) {
    extern __shared__ double big[];  // force one CTA per SM
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    unsigned long long t0, t1;
    __syncthreads();
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0)::"memory");
    const int r0 = rb + blockIdx.x * R;
    const int rows = min(R, n - r0);
    const int R2 = (rows + 1) / 2;
    const int t = threadIdx.x - 32;  // 15 GEMV warps (warp 0 idle, as in the panel)
    double2 acc = make_double2(0.0, 0.0);
    if (t >= 0 && rows > 0) {
        int R2p = 1;
        while (R2p < R2 && R2p < 32) R2p *= 2;
        if (R2 > 32) R2p = R2;
        const int ncl = 480 / R2p;
        const int rp = t % R2p, cl = t / R2p;
        if (rp < R2 && cl < ncl) {
            const double2 *A2 = reinterpret_cast<const double2 *>(A + r0) + rp;
            const int64_t ld2 = ld / 2;
            for (int c0 = cb + cl; c0 < n; c0 += 12 * ncl) {
                double2 v[12];
                double xv[12];
#pragma unroll
                for (int u = 0; u < 12; u++) {
                    const int c = c0 + u * ncl;
                    v[u] = c < n ? A2[c * ld2] : make_double2(0.0, 0.0);
                    xv[u] = c < n ? x[c] : 0.0;
                }
#pragma unroll
                for (int u = 0; u < 12; u++) {
                    acc.x += v[u].x * xv[u];
                    acc.y += v[u].y * xv[u];
                }
            }
        }
    }
    __syncthreads();
    if (acc.x == 1234.5) y[1] = acc.x;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1)::"memory");
    if (acc.x == 1234.5) y[0] = acc.y;
    if (threadIdx.x == 0) {
        rec[2 * blockIdx.x] = smid;
        rec[2 * blockIdx.x + 1] = t1 - t0;
    }
    if (threadIdx.x == 0 && n < 0) big[0] = 1.0;
}

__global__ void k_fill(double *a, size_t m) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < m; i += (size_t)gridDim.x * blockDim.x) {
        unsigned long long z = i * 0x9E3779B97F4A7C15ull + 0x632BE59BD9B4E019ull;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        a[i] = (double)((z ^ (z >> 31)) >> 11) * 0x1.0p-53;
    }
}

int main(int argc, char **argv) {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const int n = 16384;
    const int64_t ld = argc > 1 ? atoll(argv[1]) : n;
    double *A, *x, *y;
    unsigned long long *rec;
    cudaMalloc(&A, (size_t)ld * n * sizeof(double));
    cudaMalloc(&x, n * sizeof(double));
    cudaMalloc(&y, 64);
    cudaMalloc(&rec, 2 * nsm * sizeof(unsigned long long));
    k_fill<<<4096, 256>>>(A, (size_t)ld * n);  // random-looking data (no compressible zero pages)
    k_fill<<<64, 256>>>(x, (size_t)n);
    const size_t smem = 150 * 1024;
    cudaFuncSetAttribute(k_slab, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const int rb = argc > 3 ? atoi(argv[3]) : 0, cb = argc > 4 ? atoi(argv[4]) : 0;
    int R = (n - rb + nsm - 1) / nsm;
    R += R & 1;
    const int L = 8;
    std::vector<std::vector<double>> span(L, std::vector<double>(nsm, 0.0));
    std::vector<unsigned long long> h(2 * nsm);
    for (int l = 0; l < L; l++) {
        k_slab<<<nsm, 512, smem>>>(A, n, ld, R, x, y, rec, rb, cb);
        cudaMemcpy(h.data(), rec, h.size() * 8, cudaMemcpyDeviceToHost);
        for (int b = 0; b < nsm; b++) span[l][h[2 * b]] = h[2 * b + 1] / 1e3;  // by SM id, microseconds
        if (l == L - 1 && argc > 5) {  // per CTA (block index order)
            printf("by CTA: ");
            for (int b = 0; b < nsm; b++) printf("%d:%.0f ", b, h[2 * b + 1] / 1e3);
            printf("\n");
        }
    }
    for (int l = 0; l < L; l++) {
        double mn = 1e30, mx = 0, s = 0;
        for (int q = 0; q < nsm; q++) {
            mn = std::fmin(mn, span[l][q]);
            mx = std::fmax(mx, span[l][q]);
            s += span[l][q];
        }
        printf("launch %d: per-SM span min %.1f mean %.1f max %.1f us (max/mean %.3f), %.0f GB/s at the max span\n", l, mn,
               s / nsm, mx, mx / (s / nsm), (double)n * n * 8 / (mx * 1e3));
    }
    // correlation of the per-SM spans between launches l and l+1 (launch 0 = warm-up)
    for (int l = 1; l + 1 < L; l++) {
        double ma = 0, mb = 0;
        for (int q = 0; q < nsm; q++) {
            ma += span[l][q];
            mb += span[l + 1][q];
        }
        ma /= nsm;
        mb /= nsm;
        double sab = 0, saa = 0, sbb = 0;
        for (int q = 0; q < nsm; q++) {
            sab += (span[l][q] - ma) * (span[l + 1][q] - mb);
            saa += (span[l][q] - ma) * (span[l][q] - ma);
            sbb += (span[l + 1][q] - mb) * (span[l + 1][q] - mb);
        }
        printf("corr(launch %d, launch %d) over SMs: %.3f\n", l, l + 1, sab / std::sqrt(saa * sbb));
    }
    // mean span per SM over launches 1..L-1, printed by SM id (for a static weighting table)
    printf("ld = %lld rows %d.. cols %d.. R = %d\n", (long long)ld, rb, cb, R);
    if (argc > 2) return 0;
    printf("per-SM mean span (us), by smid:\n");
    for (int q = 0; q < nsm; q++) {
        double s = 0;
        for (int l = 1; l < L; l++) s += span[l][q];
        printf("%.0f%s", s / (L - 1), (q % 16 == 15) ? "\n" : " ");
    }
    printf("\nerr: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
