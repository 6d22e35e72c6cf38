// Microbenchmark: attainable HBM READ bandwidth for the panel GEMV's access pattern, next to a
// flat streaming read (the panel kernel is ~all reads; MEASURED_PEAKS' hbm_gbs is a copy).
//   flat:   grid-stride double2 loads over 2 GiB (sum kept live)
//   slab:   y = A x on a column-major n x n matrix, CTA b owns rows [b R, (b+1) R) of every
//           column (the panel GEMV's row partition): per column a contiguous 8 R-byte segment
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/mb_read scripts/mb_read.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_flat(const double2 *__restrict__ a, size_t n2, double *out) {
    double s = 0.0;
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n2; i += (size_t)gridDim.x * blockDim.x) {
        const double2 v = __ldcs(a + i);
        s += v.x + v.y;
    }
    if (s == 1234.5) out[0] = s;
}

// rows per CTA R (even), lanes: R/2 lanes per column (double2 pairs), columns strided over the
// CTA's remaining lane groups; 8 loads in flight per lane
template <int NT>
__global__ void __launch_bounds__(NT) k_slab(const double *__restrict__ A, int n, int64_t ld, int R,
                                             const double *__restrict__ x, double *y) {
    const int r0 = blockIdx.x * R;
    const int rows = min(R, n - r0);
    if (rows <= 0) return;
    const int R2 = (rows + 1) / 2;
    const int lanes_per_col = R2;
    const int ncl = NT / lanes_per_col;
    const int t = threadIdx.x, rp = t % lanes_per_col, cl = t / lanes_per_col;
    double2 acc = make_double2(0.0, 0.0);
    if (cl < ncl) {
        const double2 *A2 = reinterpret_cast<const double2 *>(A + r0) + rp;
        const int64_t ld2 = ld / 2;
        for (int c0 = cl; c0 < n; c0 += 8 * ncl) {
            double2 v[8];
            double xv[8];
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int c = c0 + u * ncl;
                v[u] = c < n ? __ldcs(A2 + c * ld2) : make_double2(0.0, 0.0);
                xv[u] = c < n ? x[c] : 0.0;
            }
#pragma unroll
            for (int u = 0; u < 8; u++) {
                acc.x += v[u].x * xv[u];
                acc.y += v[u].y * xv[u];
            }
        }
    }
    if (acc.x == 1234.5) y[r0 + 2 * rp] = acc.x + acc.y;
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const int n = 16384;
    const int64_t ld = n;
    double *A, *x, *y, *out;
    cudaMalloc(&A, (size_t)ld * n * sizeof(double));
    cudaMalloc(&x, n * sizeof(double));
    cudaMalloc(&y, n * sizeof(double));
    cudaMalloc(&out, 64);
    cudaMemset(A, 0, (size_t)ld * n * sizeof(double));
    cudaMemset(x, 0, n * sizeof(double));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const double bytes = (double)ld * n * 8;
    for (int bpsm : {1, 2, 4, 8}) {
        float best = 1e30f;
        for (int rep = 0; rep < 5; rep++) {
            cudaEventRecord(e0);
            k_flat<<<nsm * bpsm, 512>>>(reinterpret_cast<const double2 *>(A), (size_t)ld * n / 2, out);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        printf("flat read  %d x 512 threads per SM: %7.1f GB/s\n", bpsm, bytes / best / 1e6);
    }
    // the panel GEMV partition: nsm CTAs x 512 threads, R = ceil(n / nsm) rounded to even
    for (int cols_frac : {1, 2, 4}) {
        const int nn = n / cols_frac;  // trailing block nn x nn (early / later panels)
        int R = (nn + nsm - 1) / nsm;
        R += R & 1;
        float best = 1e30f;
        for (int rep = 0; rep < 5; rep++) {
            cudaEventRecord(e0);
            k_slab<512><<<nsm, 512>>>(A, nn, ld, R, x, y);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        printf("slab GEMV  %d x %d block (ld %lld), R = %d rows per CTA: %7.1f GB/s\n", nn, nn, (long long)ld, R,
               (double)nn * nn * 8 / best / 1e6);
    }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
