// ft_abft.cu -- checksum encode / verify / locate / correct / inject kernels and
// small utilities of the product path.
//
//   encode            r = A e, c = e^T A, kappa = e^T A e      P:218-224 (Sec. IV-B, Fig. 3), R22
//   pre-update check  e^T Y vs Y_chk, e^T V vs V_chk             R15 (extends Alg. 3 l.6-7)
//   end check         |sum r - kappa|, |sum c - kappa|           P:256-260 (Alg. 3 l.12-13), R11
//   full verify       D_r = r - L e, D_c = c - e^T L             P:272 (Sec. IV-F, location)
//   fix               A(i,j) = r(i) - sum_{k!=j} A(i,k) (or col)
//   inject            XOR one bit of a binary64 word             P:48-52 failure model, R16
#include <algorithm>

#include "ft_common.cuh"
#include "ft_internal.h"

static const double EPS = 2.220446049250313e-16;

__global__ void k_copy_in(const double *__restrict__ A, int lda, double *__restrict__ Aw, int64_t ldw, int n) {
    int64_t j = blockIdx.y;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        Aw[i + j * ldw] = A[i + j * (int64_t)lda];
}
cudaError_t ft_copy_in(const double *A, int lda, double *Aw, int64_t ldw, int n, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    g_ft_launches++;
    k_copy_in<<<dim3((n + 255) / 256 < 8 ? (n + 255) / 256 : 8, n), 256, 0, s>>>(A, lda, Aw, ldw, n);
    return cudaGetLastError();
}
__global__ void k_copy_out(const double *__restrict__ Aw, int64_t ldw, double *__restrict__ A, int lda, int n) {
    int64_t j = blockIdx.y;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        A[i + j * (int64_t)lda] = Aw[i + j * ldw];
}
// symmetric input (ft_dsytrd, uplo 'L'): the working copy's strict upper triangle from the lower one
__global__ void k_mirror_lower(double *Aw, int64_t ldw, int n) {
    const int64_t j = blockIdx.y;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < j; i += gridDim.x * blockDim.x)
        Aw[i + j * ldw] = Aw[j + (int64_t)i * ldw];
}
cudaError_t ft_mirror_lower(double *Aw, int64_t ldw, int n, cudaStream_t s) {
    if (n <= 1) return cudaSuccess;
    g_ft_launches++;
    k_mirror_lower<<<dim3((n + 255) / 256 < 8 ? (n + 255) / 256 : 8, n), 256, 0, s>>>(Aw, ldw, n);
    return cudaGetLastError();
}
// copy-out of the lower triangle only (the caller's strict upper part is not referenced), and the
// tridiagonal's diagonal d and subdiagonal e
__global__ void k_copy_out_lower(const double *__restrict__ Aw, int64_t ldw, double *__restrict__ A, int lda, int n,
                                 double *d, double *e) {
    const int64_t j = blockIdx.y;
    for (int i = (int)j + blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        const double v = Aw[i + j * ldw];
        A[i + j * (int64_t)lda] = v;
        if (i == j) d[i] = v;
        else if (i == j + 1) e[j] = v;
    }
}
cudaError_t ft_copy_out_lower(const double *Aw, int64_t ldw, double *A, int lda, int n, double *d, double *e,
                              cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    g_ft_launches++;
    k_copy_out_lower<<<dim3((n + 255) / 256 < 8 ? (n + 255) / 256 : 8, n), 256, 0, s>>>(Aw, ldw, A, lda, n, d, e);
    return cudaGetLastError();
}
cudaError_t ft_copy_out(const double *Aw, int64_t ldw, double *A, int lda, int n, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    g_ft_launches++;
    k_copy_out<<<dim3((n + 255) / 256 < 8 ? (n + 255) / 256 : 8, n), 256, 0, s>>>(Aw, ldw, A, lda, n);
    return cudaGetLastError();
}

// control block initialisation as a kernel (capturable into a CUDA graph)
__global__ void k_ctl_init(FtCtl *ctl, double c_thr) {
    unsigned *w = reinterpret_cast<unsigned *>(ctl);
    for (size_t i = threadIdx.x; i < sizeof(FtCtl) / sizeof(unsigned); i += blockDim.x) w[i] = 0u;
    __syncthreads();
    if (threadIdx.x == 0) ctl->c_thr = c_thr;
}
cudaError_t ft_ctl_init(FtCtl *ctl, double c_thr, cudaStream_t s) {
    g_ft_launches++;
    k_ctl_init<<<1, 256, 0, s>>>(ctl, c_thr);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// encode: row sums as 2-D tiled partial sums (thread per row, 64-column chunks, fixed-order
// finish: deterministic), column sums (warp per column), ||A||_F^2
// ---------------------------------------------------------------------------
#define LS_RB 256  // rows per block of the row-sum passes
static int ls_chunks(int n) {  // column chunks (<= 64): partials fit the 64 x ldw scratch
    int cb = (n + 63) / 64;
    if (cb < 32) cb = 32;
    return (n + cb - 1) / cb;
}
// rowpart[chunk][i] = sum_{j in chunk} w(i,j) A(i,j), w = 1 (mode -1: encode), the logical-H
// mask (mode 0) or the Householder-vector mask (mode 1); sq_part[block] = sum A^2 (encode)
__device__ __forceinline__ bool in_v(int i, int j, int ilo, int ihi, int cdone) {
    return j >= ilo - 1 && j < cdone && j <= ihi - 2 && i >= j + 2 && i < ihi;
}
__global__ void __launch_bounds__(LS_RB) k_rowsum_part(const double *__restrict__ Aw, int64_t ldw, int n, int nchunk,
                                                       int mode, int ilo, int ihi, int cdone, double *rowpart,
                                                       double *sq_part, int wgt = 0) {
    const int i = blockIdx.x * LS_RB + threadIdx.x;
    const int cw = (n + nchunk - 1) / nchunk;
    const int j0 = blockIdx.y * cw, j1 = min(n, j0 + cw);
    double s = 0.0, q = 0.0;
    if (i < n && wgt) {  // weighted pair (NEXT-1): sum_j w_j A(i, j), w_j = j + 1
        const double *a = Aw + i;
        for (int j = j0; j < j1; j++) {
            const bool v = mode >= 0 && in_v(i, j, ilo, ihi, cdone);
            if (mode < 0 || (mode == 0 ? !v : v)) s += a[(int64_t)j * ldw] * (double)(j + 1);
        }
        rowpart[(int64_t)blockIdx.y * n + i] = s;
    } else if (i < n) {
        const double *a = Aw + i;
        if (mode < 0) {
#pragma unroll 8
            for (int j = j0; j < j1; j++) {
                const double x = a[(int64_t)j * ldw];
                s += x;
                q += x * x;
            }
        } else {
#pragma unroll 8
            for (int j = j0; j < j1; j++) {
                const bool v = in_v(i, j, ilo, ihi, cdone);
                if (mode == 0 ? !v : v) s += a[(int64_t)j * ldw];
            }
        }
        rowpart[(int64_t)blockIdx.y * n + i] = s;
    }
    if (sq_part) {
        q = warp_sum(q);
        __shared__ double ws[LS_RB / 32];
        if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = q;
        __syncthreads();
        if (threadIdx.x == 0) {
            double t = 0.0;
            for (int w = 0; w < LS_RB / 32; w++) t += ws[w];
            sq_part[blockIdx.y * gridDim.x + blockIdx.x] = t;
        }
    }
}
// out[i * oinc] = (base ? base[i * binc] : 0) - / + sum_chunk rowpart[chunk][i]
__global__ void k_rowsum_finish(const double *rowpart, int n, int nchunk, const double *base, int64_t binc,
                                double *out, int64_t oinc) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    double s = 0.0;
    for (int c = 0; c < nchunk; c++) s += rowpart[(int64_t)c * n + i];
    out[(int64_t)i * oinc] = base ? base[(int64_t)i * binc] - s : s;
}
__global__ void k_encode_cols(double *Aw, int64_t ldw, int n) {
    int j = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    int lane = threadIdx.x & 31;
    if (j >= n) return;
    double s = 0.0;
    for (int i = lane; i < n; i += 32) s += Aw[i + (int64_t)j * ldw];
    s = warp_sum(s);
    if (lane == 0) Aw[n + (int64_t)j * ldw] = s;  // c(j) in row n
}
__global__ void k_encode_finish(double *Aw, int64_t ldw, int n, const double *sq_part, int nparts, FtCtl *ctl) {
    // kappa = sum r, ||A||_F^2 = sum of the squares' partials (both in a fixed order: strided
    // per thread, then warps, then thread 0 over the warps)
    __shared__ double ws[32], wq[32];
    double s = 0.0, q = 0.0;
    for (int i = threadIdx.x; i < n; i += blockDim.x) s += Aw[i + (int64_t)n * ldw];
    for (int b = threadIdx.x; b < nparts; b += blockDim.x) q += sq_part[b];
    s = warp_sum(s);
    q = warp_sum(q);
    if ((threadIdx.x & 31) == 0) {
        ws[threadIdx.x >> 5] = s;
        wq[threadIdx.x >> 5] = q;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double k = 0.0, qq = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
            k += ws[w];
            qq += wq[w];
        }
        Aw[n + (int64_t)n * ldw] = k;
        ctl->normF = sqrt(qq);
    }
}
// frozen row sums before the first panel: columns 0..ilo-2 are final (R5/R6)
__global__ void k_frozen_init(const double *Aw, int64_t ldw, int n, int ncols, double *Fr) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    double s = 0.0;
    for (int j = 0; j < ncols; j++) s += Aw[i + (int64_t)j * ldw];
    Fr[i] = s;
}
cudaError_t ft_frozen_init(const double *Aw, int64_t ldw, int n, int ncols, double *Fr, cudaStream_t s) {
    g_ft_launches++;
    k_frozen_init<<<(n + 255) / 256, 256, 0, s>>>(Aw, ldw, n, ncols, Fr);
    return cudaGetLastError();
}
cudaError_t ft_encode(double *Aw, int64_t ldw, int n, FtCtl *ctl, double *scratch, double *linepart,
                      cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    const int nrb = (n + LS_RB - 1) / LS_RB, nch = ls_chunks(n);
    g_ft_launches += 4;
    k_rowsum_part<<<dim3(nrb, nch), LS_RB, 0, s>>>(Aw, ldw, n, nch, -1, 0, 0, 0, linepart, scratch);
    k_rowsum_finish<<<(n + 255) / 256, 256, 0, s>>>(linepart, n, nch, nullptr, 0, Aw + (int64_t)n * ldw, 1);
    k_encode_cols<<<(n + 7) / 8, 256, 0, s>>>(Aw, ldw, n);
    k_encode_finish<<<1, 1024, 0, s>>>(Aw, ldw, n, scratch, nrb * nch, ctl);
    return cudaGetLastError();
}

// ||A||_F only (ABFT off still reports drift in units of ||A||_F)
__global__ void k_frob(const double *A, int lda, int n, FtCtl *ctl) {
    __shared__ double ws[32];
    double q = 0.0;
    for (int64_t idx = threadIdx.x; idx < (int64_t)n * n; idx += blockDim.x) {
        double a = A[(idx % n) + (idx / n) * (int64_t)lda];
        q += a * a;
    }
    q = warp_sum(q);
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = q;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) t += ws[w];
        ctl->normF = sqrt(t);
    }
}
cudaError_t ft_frob_to_ctl(const double *A, int lda, int n, FtCtl *ctl, cudaStream_t s) {
    g_ft_launches++;
    k_frob<<<1, 1024, 0, s>>>(A, lda, n, ctl);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// pre-update check sums: eY(j) = sum_{i<ihi} Y(i,j), eV(j) = sum_{k+1<=i<ihi} V(i,j)
// (computed after the AFTER_PANEL injection point; reading R15)
// ---------------------------------------------------------------------------
__global__ void k_precheck(const double *Y, const double *V, int64_t ldw, int ihi, int k, int ib, FtCtl *ctl) {
    if (ctl->halt) return;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int rows_per = 256;
    const int i0 = blockIdx.x * rows_per, i1 = min(ihi, i0 + rows_per);
    for (int j = wid; j < ib; j += nw) {
        double sy = 0.0, sv = 0.0;
        for (int i = i0 + lane; i < i1; i += 32) {
            sy += Y[i + (int64_t)j * ldw];
            if (i >= k + 1) sv += V[i + (int64_t)j * ldw];
        }
        sy = warp_sum(sy);
        sv = warp_sum(sv);
        if (lane == 0) {
            atomicAdd(&ctl->eY[j * FT_ESTR], sy);
            atomicAdd(&ctl->eV[j * FT_ESTR], sv);
        }
    }
}
cudaError_t ft_precheck(const double *Y, const double *V, int64_t ldw, int n, int ihi, int k, int ib,
                        FtCtl *ctl, cudaStream_t s) {
    int nblk = (ihi + 255) / 256;
    g_ft_launches++;
    k_precheck<<<nblk, 512, 0, s>>>(Y, V, ldw, ihi, k, ib, ctl);
    return cudaGetLastError();
}

// one warp: decide whether to halt before the updates consume the panel's output
__global__ void k_decide(const double *Y, const double *V, const double *T, int64_t ldw, int n, int k, int ib,
                         int panel, FtCtl *ctl) {
    if (ctl->halt) return;
    const int lane = threadIdx.x;
    const double unit = (double)n * EPS * ctl->normF;
    const double c_thr = ctl->c_thr;
    double tmax = 0.0;
    for (int i = lane; i < ib * ib; i += 32) {
        int a = i % ib, b = i / ib;
        tmax = fmax(tmax, fabs(T[a + b * FT_NBMAX]));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) tmax = fmax(tmax, __shfl_xor_sync(0xffffffffu, tmax, o));
    int reason = 0;
    if (ctl->nflag > 0) reason |= 1;
    const double tauY = c_thr * unit * (tmax > 1.0 ? tmax : 1.0);
    const double tauV = c_thr * (double)n * EPS * sqrt((double)n);
    for (int j = lane; j < ib; j += 32) {
        double dy = ctl->eY[j * FT_ESTR] - Y[n + (int64_t)j * ldw];
        double dv = ctl->eV[j * FT_ESTR] - V[n + (int64_t)j * ldw];
        if (not_within(dy, tauY)) reason |= 2;
        if (not_within(dv, tauV)) reason |= 4;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) reason |= __shfl_xor_sync(0xffffffffu, reason, o);
    __syncwarp();
    if (lane == 0) {
        if (reason) {
            ctl->halt_panel = panel;
            ctl->halt_stage = 1;
            ctl->halt_reason = reason;
            __threadfence();
            ctl->halt = 1;
        }
        ctl->nflag = 0;
    }
    for (int j = lane; j < FT_NBMAX; j += 32) {
        ctl->eY[j * FT_ESTR] = 0.0;
        ctl->eV[j * FT_ESTR] = 0.0;
    }
}
cudaError_t ft_decide(const double *Y, const double *V, const double *T, int64_t ldw, int n, int k, int ib,
                      int panel, FtCtl *ctl, cudaStream_t s) {
    g_ft_launches++;
    k_decide<<<1, 32, 0, s>>>(Y, V, T, ldw, n, k, ib, panel, ctl);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// end-of-iteration check (Alg. 3 l.12-13) + frozen-row-sum bookkeeping.
// Grid-stride blocks; the last block to finish takes the decision.
//   sum r = sum_{i<n} A(i,n), sum c = sum_{j<n} A(n,j), kappa = A(n,n)
//   Fr(i) += sum_{col in [k,e), i <= col+1} A(i,col)   for i <= e (columns frozen now)
// ---------------------------------------------------------------------------
__global__ void k_endcheck(double *Aw, int64_t ldw, int n, int ihi, int k, int ib, int panel, int policy,
                           double *Fr, FtCtl *ctl, int weighted) {
    if (ctl->halt) return;
    __shared__ double ws[4][32];
    __shared__ int last;
    double sr = 0.0, sc = 0.0, srw = 0.0, scw = 0.0;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        sr += Aw[i + (int64_t)n * ldw];
        sc += Aw[n + (int64_t)i * ldw];
        if (weighted) {  // the weighted pair's sums (NEXT-1): sum r_w = e^T L w, sum c_w = w^T L e
            srw += Aw[i + (int64_t)(n + 1) * ldw];
            scw += Aw[n + 1 + (int64_t)i * ldw];
        }
    }
    sr = warp_sum(sr);
    sc = warp_sum(sc);
    srw = warp_sum(srw);
    scw = warp_sum(scw);
    if ((threadIdx.x & 31) == 0) {
        ws[0][threadIdx.x >> 5] = sr;
        ws[1][threadIdx.x >> 5] = sc;
        ws[2][threadIdx.x >> 5] = srw;
        ws[3][threadIdx.x >> 5] = scw;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double a = 0.0, b = 0.0, c2 = 0.0, d2 = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
            a += ws[0][w];
            b += ws[1][w];
            c2 += ws[2][w];
            d2 += ws[3][w];
        }
        atomicAdd(&ctl->sums[0], a);
        atomicAdd(&ctl->sums[1], b);
        if (weighted) {
            atomicAdd(&ctl->wsums[0], c2);
            atomicAdd(&ctl->wsums[1], d2);
        }
        last = (atom_add_acqrel_s32(&ctl->done_count, 1) == (int)gridDim.x - 1);
    }
    __syncthreads();
    if (!last) return;
    if (threadIdx.x == 0) {
        double Sr = atomicAdd(&ctl->sums[0], 0.0), Sc = atomicAdd(&ctl->sums[1], 0.0);
        double kap = Aw[n + (int64_t)n * ldw];
        double unit = (double)n * EPS * ctl->normF;
        double tauS = ctl->c_thr * unit * sqrt((double)n);
        int reason = 0;
        if (policy == FT_POLICY_PAPER) {
            if (not_within(Sr - Sc, tauS)) reason |= 8;
        } else {
            if (not_within(Sr - kap, tauS) || not_within(Sc - kap, tauS)) reason |= 8;
        }
        if (weighted) {
            const double Srw = atomicAdd(&ctl->wsums[0], 0.0), Scw = atomicAdd(&ctl->wsums[1], 0.0);
            const double krw = Aw[n + (int64_t)(n + 1) * ldw], kcw = Aw[n + 1 + (int64_t)n * ldw];
            if (not_within(Srw - krw, tauS * n) || not_within(Scw - kcw, tauS * n)) reason |= 64;
            ctl->wsums[0] = 0.0;
            ctl->wsums[1] = 0.0;
        }
        ctl->sums[0] = 0.0;
        ctl->sums[1] = 0.0;
        ctl->done_count = 0;
        if (reason) {
            ctl->halt_panel = panel;
            ctl->halt_stage = 2;
            ctl->halt_reason = reason;
            __threadfence();
            ctl->halt = 1;
        }
    }
}
// frozen row sums of the panel columns that just became final (rows 0..e; R6)
__global__ void k_frozen_rows(const double *Aw, int64_t ldw, int n, int k, int e, double *Fr, FtCtl *ctl) {
    if (ctl->halt) return;
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i > e || i >= n) return;
    double s = 0.0;
    for (int col = k; col < e; col++)
        if (i <= col + 1) s += Aw[i + (int64_t)col * ldw];
    Fr[i] += s;
}
cudaError_t ft_endcheck(double *Aw, int64_t ldw, int n, int ihi, int k, int ib, int panel, int policy,
                        double *Fr, FtCtl *ctl, cudaStream_t s, int weighted) {
    int nblk = (n + 1023) / 1024;
    if (nblk > 16) nblk = 16;
    g_ft_launches++;
    k_endcheck<<<nblk, 1024, 0, s>>>(Aw, ldw, n, ihi, k, ib, panel, policy, Fr, ctl, weighted);
    int e = k + ib;
    if (Fr) {
        g_ft_launches++;
        k_frozen_rows<<<(e + 1 + 255) / 256, 256, 0, s>>>(Aw, ldw, n, k, e, Fr, ctl);
    }
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// fault injector: XOR one bit of one binary64 word (skipped after a halt; once per fault)
// ---------------------------------------------------------------------------
__global__ void k_inject(double *addr, int fidx, int bit, FtCtl *ctl) {
    if (ctl->halt || ctl->inj_done[fidx]) return;
    unsigned long long u = __double_as_longlong(*addr);
    double old = *addr;
    u ^= 1ull << (bit & 63);
    *addr = __longlong_as_double(u);
    ctl->inj_delta[fidx] = __longlong_as_double(u) - old;
    ctl->inj_done[fidx] = 1;
}
cudaError_t ft_inject(double *addr, int fidx, int bit, FtCtl *ctl, cudaStream_t s) {
    g_ft_launches++;
    k_inject<<<1, 1, 0, s>>>(addr, fidx, bit, ctl);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// full verification over the logical matrix (recovery path and final check).
// mode 0 (H): L(i,j) = 0 for stored Householder vectors (j in [ilo-1, cdone), j <= ihi-2,
//             j+2 <= i < ihi), else A(i,j).  r/c are the maintained checksums.
// mode 1 (Q): L(i,j) = A(i,j) exactly on that V region, 0 elsewhere; r/c = Qr/Qc.
// Fr (mode 0, optional) is ignored here: the full verify recomputes everything.
// sums[0] = sum r, sums[1] = sum c.
// ---------------------------------------------------------------------------
__global__ void k_fv_cols(const double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode,
                          const double *c, int64_t cinc, double *Dc, int wgt = 0) {
    int j = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    int lane = threadIdx.x & 31;
    if (j >= n) return;
    double s = 0.0;
    for (int i = lane; i < n; i += 32) {
        bool v = in_v(i, j, ilo, ihi, cdone);
        if (mode == 0 ? !v : v) s += wgt ? (double)(i + 1) * Aw[i + (int64_t)j * ldw] : Aw[i + (int64_t)j * ldw];
    }
    s = warp_sum(s);
    if (lane == 0) Dc[j] = c[(int64_t)j * cinc] - s;
}
__global__ void k_fv_sums(int n, const double *r, int64_t rinc, const double *c, int64_t cinc, double *sums) {
    __shared__ double ws[2][32];
    double a = 0.0, b = 0.0;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
        a += r[(int64_t)i * rinc];
        b += c[(int64_t)i * cinc];
    }
    a = warp_sum(a);
    b = warp_sum(b);
    if ((threadIdx.x & 31) == 0) {
        ws[0][threadIdx.x >> 5] = a;
        ws[1][threadIdx.x >> 5] = b;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double x = 0.0, y = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
            x += ws[0][w];
            y += ws[1][w];
        }
        sums[0] = x;
        sums[1] = y;
    }
}
cudaError_t ft_full_verify(const double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode,
                           const double *r, int64_t rinc, const double *c, int64_t cinc, const double *Fr,
                           double *Dr, double *Dc, double *sums, double *linepart, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    g_ft_launches += 4;
    const int nrb = (n + LS_RB - 1) / LS_RB, nch = ls_chunks(n);
    k_rowsum_part<<<dim3(nrb, nch), LS_RB, 0, s>>>(Aw, ldw, n, nch, mode, ilo, ihi, cdone, linepart, nullptr);
    k_rowsum_finish<<<(n + 255) / 256, 256, 0, s>>>(linepart, n, nch, r, rinc, Dr, 1);
    k_fv_cols<<<(n + 7) / 8, 256, 0, s>>>(Aw, ldw, n, ilo, ihi, cdone, mode, c, cinc, Dc);
    k_fv_sums<<<1, 1024, 0, s>>>(n, r, rinc, c, cinc, sums);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// Weighted checksum pair (NEXT-1; w_i = i + 1), opts.weighted = 1.  Column n+1 of the
// working array is r_w = L w, row n+1 is c_w = w^T L; (n, n+1) = e^T L w, (n+1, n) = w^T L e,
// (n+1, n+1) = w^T L w.  They ride through the update GEMMs as one more row / column (Theorem 1 holds
// for any weight vector); the panel's rows n+1 of V and Y (w^T V and c_w V T) are formed
// after the panel by k_wchk_*; the finished panel columns' c_w entries are re-encoded (k_cw_panel).
// ---------------------------------------------------------------------------
// corners of the weighted pair after encode: (n, n+1) = sum r_w, (n+1, n) = sum c_w, (n+1, n+1) = sum w_j c_w(j)
__global__ void k_encode_w_finish(double *Aw, int64_t ldw, int n) {
    __shared__ double ws[3][32];
    double a = 0.0, b = 0.0, c = 0.0;
    const double *rw = Aw + (int64_t)(n + 1) * ldw;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
        a += rw[i];
        const double cwj = Aw[n + 1 + (int64_t)i * ldw];
        b += cwj;
        c += (double)(i + 1) * cwj;
    }
    a = warp_sum(a);
    b = warp_sum(b);
    c = warp_sum(c);
    if ((threadIdx.x & 31) == 0) {
        ws[0][threadIdx.x >> 5] = a;
        ws[1][threadIdx.x >> 5] = b;
        ws[2][threadIdx.x >> 5] = c;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double x = 0.0, y = 0.0, z = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
            x += ws[0][w];
            y += ws[1][w];
            z += ws[2][w];
        }
        Aw[n + (int64_t)(n + 1) * ldw] = x;
        Aw[n + 1 + (int64_t)n * ldw] = y;
        Aw[n + 1 + (int64_t)(n + 1) * ldw] = z;
    }
}
// c_w(j) = sum_i w_i A(i, j) into row n+1 (warp per column, fixed order)
__global__ void k_encode_cols_w(double *Aw, int64_t ldw, int n) {
    int j = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    int lane = threadIdx.x & 31;
    if (j >= n) return;
    double s = 0.0;
    for (int i = lane; i < n; i += 32) s += (double)(i + 1) * Aw[i + (int64_t)j * ldw];
    s = warp_sum(s);
    if (lane == 0) Aw[n + 1 + (int64_t)j * ldw] = s;
}
cudaError_t ft_encode_w(double *Aw, int64_t ldw, int n, double *linepart, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    const int nrb = (n + LS_RB - 1) / LS_RB, nch = ls_chunks(n);
    g_ft_launches += 4;
    k_rowsum_part<<<dim3(nrb, nch), LS_RB, 0, s>>>(Aw, ldw, n, nch, -1, 0, 0, 0, linepart, nullptr, 1);
    k_rowsum_finish<<<(n + 255) / 256, 256, 0, s>>>(linepart, n, nch, nullptr, 0, Aw + (int64_t)(n + 1) * ldw, 1);
    k_encode_cols_w<<<(n + 7) / 8, 256, 0, s>>>(Aw, ldw, n);
    k_encode_w_finish<<<1, 1024, 0, s>>>(Aw, ldw, n);
    return cudaGetLastError();
}

// weighted syndromes of the full verification: D_rw = r_w - L w, D_cw = c_w - w^T L (mode 0, H logical)
cudaError_t ft_full_verify_w(const double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, const double *rw,
                             const double *cw, int64_t cinc, double *Drw, double *Dcw, double *linepart,
                             cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    g_ft_launches += 3;
    const int nrb = (n + LS_RB - 1) / LS_RB, nch = ls_chunks(n);
    k_rowsum_part<<<dim3(nrb, nch), LS_RB, 0, s>>>(Aw, ldw, n, nch, 0, ilo, ihi, cdone, linepart, nullptr, 1);
    k_rowsum_finish<<<(n + 255) / 256, 256, 0, s>>>(linepart, n, nch, rw, 1, Drw, 1);
    k_fv_cols<<<(n + 7) / 8, 256, 0, s>>>(Aw, ldw, n, ilo, ihi, cdone, 0, cw, cinc, Dcw, 1);
    return cudaGetLastError();
}

// after the panel: V(n+1, j) = sum_i w_i V(i, j) and s(j) = sum_i c_w0(i) V(i, j) over the reflector
// rows k+1 .. ihi-1 (c_w0 = row n+1 at panel start: the panel does not touch it), as per-chunk partials
#define WCHK_ROWS 256
__global__ void __launch_bounds__(256) k_wchk_part(const double *Aw, int64_t ldw, const double *V, int n, int ihi,
                                                   int k, int ib, double *part, const FtCtl *ctl) {
    if (ctl->halt) return;
    const int j = threadIdx.x & 63, q = threadIdx.x >> 6;  // 4 row phases x 64 columns
    const int r0 = k + 1 + blockIdx.x * WCHK_ROWS, r1 = min(ihi, r0 + WCHK_ROWS);
    double sw = 0.0, sc = 0.0;
    if (j < ib)
        for (int i = r0 + q; i < r1; i += 4) {
            const double v = V[i + (int64_t)j * ldw];
            sw += (double)(i + 1) * v;
            sc += Aw[n + 1 + (int64_t)i * ldw] * v;
        }
    __shared__ double red[2][4][64];
    red[0][q][j] = sw;
    red[1][q][j] = sc;
    __syncthreads();
    if (q == 0) {
        part[(int64_t)blockIdx.x * 128 + j] = ((red[0][0][j] + red[0][1][j]) + (red[0][2][j] + red[0][3][j]));
        part[(int64_t)blockIdx.x * 128 + 64 + j] = ((red[1][0][j] + red[1][1][j]) + (red[1][2][j] + red[1][3][j]));
    }
}
// chunk partials in chunk order; V(n+1, :) = w^T V, Y(n+1, :) = (c_w0 V) T  (Y = A V T, DLAHR2)
__global__ void k_wchk_finish(double *V, double *Y, const double *T, int64_t ldw, int n, int ib, const double *part,
                              int nchunk, const FtCtl *ctl) {
    if (ctl->halt) return;
    __shared__ double sc[64];
    const int j = threadIdx.x;
    double a = 0.0, b = 0.0;
    for (int c = 0; c < nchunk; c++) {
        a += part[(int64_t)c * 128 + j];
        b += part[(int64_t)c * 128 + 64 + j];
    }
    sc[j] = b;
    __syncthreads();
    if (j < ib) {
        double y = 0.0;
        for (int bb = 0; bb <= j; bb++) y += sc[bb] * T[bb + j * FT_NBMAX];
        V[n + 1 + (int64_t)j * ldw] = a;
        Y[n + 1 + (int64_t)j * ldw] = y;
    }
}
cudaError_t ft_wchk(const double *Aw, double *V, double *Y, const double *T, int64_t ldw, int n, int ihi, int k,
                    int ib, double *part, const FtCtl *ctl, cudaStream_t s) {
    const int nchunk = std::max(1, (ihi - k - 1 + WCHK_ROWS - 1) / WCHK_ROWS);
    g_ft_launches += 2;
    k_wchk_part<<<nchunk, 256, 0, s>>>(Aw, ldw, V, n, ihi, k, ib, part, ctl);
    k_wchk_finish<<<1, 64, 0, s>>>(V, Y, T, ldw, n, ib, part, nchunk, ctl);
    return cudaGetLastError();
}

// the finished panel columns [k, e): c_w(col) re-encoded from the logical column (rows outside the
// stored Householder vectors; R6), once the iteration has made them final
__global__ void k_cw_panel(double *Aw, int64_t ldw, int n, int ilo, int ihi, int k, int e, const FtCtl *ctl) {
    if (ctl->halt) return;
    const int col = k + blockIdx.x;
    if (col >= e) return;
    __shared__ double ws[32];
    double s = 0.0;
    for (int i = threadIdx.x; i < n; i += blockDim.x)
        if (!in_v(i, col, ilo, ihi, e)) s += (double)(i + 1) * Aw[i + (int64_t)col * ldw];
    s = warp_sum(s);
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) t += ws[w];
        Aw[n + 1 + (int64_t)col * ldw] = t;
    }
}
cudaError_t ft_cw_panel(double *Aw, int64_t ldw, int n, int ilo, int ihi, int k, int e, const FtCtl *ctl,
                        cudaStream_t s) {
    if (e <= k) return cudaSuccess;
    g_ft_launches++;
    k_cw_panel<<<e - k, 256, 0, s>>>(Aw, ldw, n, ilo, ihi, k, e, ctl);
    return cudaGetLastError();
}

// diskless checkpoint of the weighted pair: column n+1 (rows 0..n+1) and row n+1 (columns 0..n+1)
__global__ void k_ckpt_w(double *Aw, int64_t ldw, int n, double *ck, int restore, const FtCtl *ctl) {
    if (!restore && ctl->halt) return;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i <= n + 1; i += gridDim.x * blockDim.x) {
        double *a = Aw + i + (int64_t)(n + 1) * ldw, *b = Aw + n + 1 + (int64_t)i * ldw;
        if (restore) {
            *a = ck[i];
            *b = ck[n + 2 + i];
        } else {
            ck[i] = *a;
            ck[n + 2 + i] = *b;
        }
    }
}
cudaError_t ft_ckpt_w(double *Aw, int64_t ldw, int n, double *ck, int restore, const FtCtl *ctl, cudaStream_t s) {
    g_ft_launches++;
    k_ckpt_w<<<std::max(1, std::min((n + 2 + 255) / 256, 64)), 256, 0, s>>>(Aw, ldw, n, ck, restore, ctl);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// device-side decision of the final verification (a12 / P:278), fault-free path: from the full
// verification's syndromes, flag (ctl->fflag bit mode) whether anything needs the host decoder and
// record the fault-free drift; the host only looks again when a bit is set (no extra round trip)
// ---------------------------------------------------------------------------
__global__ void k_final_flags(const double *Dr, const double *Dc, const double *sums, const double *kap, int n,
                              int mode, FtCtl *ctl) {
    if (ctl->halt) return;
    __shared__ double wm[32];
    __shared__ int wf[32];
    const double unit = (double)n * EPS * (mode == 0 ? ctl->normF : sqrt((double)n));
    const double tau = ctl->c_thr * unit, tauS = tau * sqrt((double)(n > 1 ? n : 1));
    double mx = 0.0;
    int fl = 0;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
        const double a = Dr[i], b = Dc[i];
        if (not_within(a, tau)) fl = 1;
        else mx = fmax(mx, fabs(a));
        if (not_within(b, tau)) fl = 1;
        else mx = fmax(mx, fabs(b));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        fl |= __shfl_xor_sync(0xffffffffu, fl, o);
    }
    if ((threadIdx.x & 31) == 0) {
        wm[threadIdx.x >> 5] = mx;
        wf[threadIdx.x >> 5] = fl;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
            mx = fmax(mx, wm[w]);
            fl |= wf[w];
        }
        const double k = *kap;
        if (not_within(sums[0] - k, tauS) || not_within(sums[1] - k, tauS)) fl = 1;
        if (fl) ctl->fflag |= 1 << mode;
        if (mode == 0 && unit > 0.0) {
            const double rel = mx / unit;
            atomicMax(&ctl->drift_bits, (unsigned long long)__double_as_longlong(rel));
        }
    }
}
cudaError_t ft_final_flags(const double *Dr, const double *Dc, const double *sums, const double *kap, int n, int mode,
                           FtCtl *ctl, cudaStream_t s) {
    g_ft_launches++;
    k_final_flags<<<1, 1024, 0, s>>>(Dr, Dc, sums, kap, n, mode, ctl);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// R12 decoder v2 on the device (one block; written apart from the host copy in ft_driver.cu and
// from the oracle's).  Never miscorrect: refuse whenever two explanations exist.  Input: the full
// verification's syndromes D_r, D_c, the sums of r and c, kappa; output: status (0 clean, 1 fixes
// planned, 2 uncorrectable, 3 too large for the device: the host decides), the fix list (the order
// of the host decoder: data fixes, then r refreshes, then c refreshes) and the flagged counts.
// ---------------------------------------------------------------------------
#define DEC_T 256
__device__ __forceinline__ bool d_bad(double d, double tau) { return !(fabs(d) <= tau); }
__device__ __forceinline__ bool d_same(double a, double b, double tol) {
    const bool fa = isfinite(a), fb = isfinite(b);
    if (!fa || !fb) return !fa && !fb;
    return fabs(a - b) <= tol;
}
// ordered compaction of {i < n : flagged(D[i])} into out (block-wide scan over contiguous chunks)
__device__ int d_compact(const double *D, int n, double tau, int *out, int *scan) {
    const int t = threadIdx.x, chunk = (n + DEC_T - 1) / DEC_T;
    const int i0 = min(n, t * chunk), i1 = min(n, i0 + chunk);
    int c = 0;
    for (int i = i0; i < i1; i++) c += d_bad(D[i], tau);
    scan[t] = c;
    __syncthreads();
    for (int o = 1; o < DEC_T; o <<= 1) {  // inclusive Hillis-Steele scan
        const int v = t >= o ? scan[t - o] : 0;
        __syncthreads();
        scan[t] += v;
        __syncthreads();
    }
    int pos = scan[t] - c;
    for (int i = i0; i < i1; i++)
        if (d_bad(D[i], tau)) out[pos++] = i;
    __syncthreads();
    const int total = scan[DEC_T - 1];
    __syncthreads();
    return total;
}
// members of S (size m) whose syndromes add up to target (|subset| <= 3), unique; block-parallel
// over the first member.  Returns the subset size (0..3) into sub, or -1
__device__ int d_explain(const int *S, int m, const double *D, double target, double tauS, int n, int *sub,
                         int *hits, unsigned long long *best) {
    if (d_same(target, 0.0, tauS)) return 0;
    if (!isfinite(target)) {
        int k = 0;
        for (int a = 0; a < m; a++)
            if (!isfinite(D[S[a]])) {
                if (k == 3) return -1;
                sub[k++] = S[a];
            }
        return k > 0 ? k : -1;
    }
    if (m > 256) return -1;
    if (threadIdx.x == 0) {
        *hits = 0;
        *best = 0ull;
    }
    __syncthreads();
    const double e2 = 2.0 * n * EPS;
    for (int a = threadIdx.x; a < m; a += DEC_T) {
        const double da = D[S[a]];
        if (d_same(da, target, tauS + e2 * fabs(da))) {
            atomicAdd(hits, 1);
            atomicExch(best, (unsigned long long)(a + 1));
        }
        for (int b = a + 1; b < m; b++) {
            const double db = D[S[b]];
            if (d_same(da + db, target, tauS + e2 * (fabs(da) + fabs(db)))) {
                atomicAdd(hits, 1);
                atomicExch(best, (unsigned long long)(a + 1) | ((unsigned long long)(b + 1) << 20));
            }
            for (int c = b + 1; c < m; c++) {
                const double dc = D[S[c]];
                if (d_same(da + db + dc, target, tauS + e2 * (fabs(da) + fabs(db) + fabs(dc)))) {
                    atomicAdd(hits, 1);
                    atomicExch(best, (unsigned long long)(a + 1) | ((unsigned long long)(b + 1) << 20) |
                                         ((unsigned long long)(c + 1) << 40));
                }
            }
        }
    }
    __syncthreads();
    const int h = *hits;
    const unsigned long long bb = *best;
    __syncthreads();
    if (h != 1) return -1;
    int k = 0;
    for (int q = 0; q < 3; q++) {
        const int v = (int)((bb >> (20 * q)) & 0xFFFFF);
        if (v) sub[k++] = S[v - 1];
    }
    return k;
}
__global__ void __launch_bounds__(DEC_T) k_decode(const double *Dr, const double *Dc, const double *sums,
                                                  const double *kap, int n, int mode, const FtCtl *ctl, int *idx,
                                                  FtFix *fixes, int cap, FtDecOut *out) {
    __shared__ int scan[DEC_T];
    __shared__ int hits;
    __shared__ unsigned long long best;
    __shared__ int Rc[3], Cc[3], nRc, nCc;
    const double tau = ctl->c_thr * (double)n * EPS * (mode == 0 ? ctl->normF : sqrt((double)n));
    const double tauS = tau * sqrt((double)(n > 1 ? n : 1));
    int *R = idx, *C = idx + n;
    const int nR = d_compact(Dr, n, tau, R, scan);
    const int nC = d_compact(Dc, n, tau, C, scan);
    const double sr = sums[0] - *kap, sc = sums[1] - *kap;
    const bool sr0 = d_same(sr, 0.0, tauS), sc0 = d_same(sc, 0.0, tauS);
    const bool amb = !sr0 && !sc0 && d_same(sr, sc, tauS);
    if (threadIdx.x == 0) {
        out->nR = nR;
        out->nC = nC;
        out->nfix = 0;
        out->status = 2;
    }
    if (nR == 0 && nC == 0) {
        if (threadIdx.x == 0) {
            if (sr0 && sc0) out->status = 0;
            else if (amb) {  // only the corner: both sums off by the same amount
                fixes[0] = FtFix{-1, -1, 4, 0};
                out->nfix = 1;
                out->status = 1;
            }
        }
        return;
    }
    if (amb) return;  // equally explained by "corner + data errors": refuse
    {
        int sub[3];
        const int k1 = d_explain(R, nR, Dr, sr, tauS, n, sub, &hits, &best);
        if (threadIdx.x == 0) {
            nRc = k1;
            for (int q = 0; q < 3; q++) Rc[q] = q < k1 ? sub[q] : -1;
        }
        __syncthreads();
        const int k2 = d_explain(C, nC, Dc, sc, tauS, n, sub, &hits, &best);
        if (threadIdx.x == 0) {
            nCc = k2;
            for (int q = 0; q < 3; q++) Cc[q] = q < k2 ? sub[q] : -1;
        }
        __syncthreads();
    }
    if (threadIdx.x != 0) return;
    if (nRc < 0 || nCc < 0) return;
    auto inset = [](int v, const int *s3, int m) {
        for (int q = 0; q < m; q++)
            if (s3[q] == v) return true;
        return false;
    };
    int rc[3] = {Rc[0], Rc[1], Rc[2]}, cc[3] = {Cc[0], Cc[1], Cc[2]};
    int nrc = nRc, ncc = nCc;
    int nRd = 0, nCd = 0;
    for (int a = 0; a < nR; a++) nRd += !inset(R[a], rc, nrc);
    for (int b = 0; b < nC; b++) nCd += !inset(C[b], cc, ncc);
    // a flagged line without a flagged partner is a checksum word whose syndrome hid inside the
    // sum tolerance (tau < |d| <= tau sqrt(n)): accept if the whole set explains s_r / s_c
    auto whole_set = [&](const int *S, int m, const double *D, double target) {
        if (m > 3) return false;
        double sum = 0.0, sa = 0.0;
        for (int a = 0; a < m; a++) {
            const double d = D[S[a]];
            if (!(fabs(d) <= tauS)) return false;
            sum += d;
            sa += fabs(d);
        }
        return d_same(sum, target, tauS + 2.0 * n * EPS * sa);
    };
    if (nRd > 0 && nCd == 0 && whole_set(R, nR, Dr, sr)) {
        nrc = nR;
        for (int a = 0; a < nR; a++) rc[a] = R[a];
        nRd = 0;
    }
    if (nCd > 0 && nRd == 0 && whole_set(C, nC, Dc, sc)) {
        ncc = nC;
        for (int b = 0; b < nC; b++) cc[b] = C[b];
        nCd = 0;
    }
    if ((nRd == 0) != (nCd == 0)) return;
    int nf = 0;
    auto push = [&](int64_t i, int64_t j, int kind) {
        if (nf < cap) fixes[nf] = FtFix{i, j, kind, 0};
        nf++;
    };
    auto pair_tol = [&](double a, double b) { return 2.0 * tau + 2.0 * n * EPS * (fabs(a) + fabs(b)); };
    // the data rows / columns (flagged, not checksum words), in index order
    auto nth_d = [&](const int *S, int m, const int *s3, int m3, int q) {
        for (int a = 0, c = 0; a < m; a++)
            if (!inset(S[a], s3, m3)) {
                if (c == q) return S[a];
                c++;
            }
        return -1;
    };
    if (nRd > 0) {
        if (nRd == 1 && nCd == 1) {
            const int i = nth_d(R, nR, rc, nrc, 0), j = nth_d(C, nC, cc, ncc, 0);
            if (!d_same(Dr[i], Dc[j], pair_tol(Dr[i], Dc[j]))) return;
            push(i, j, 0);
        } else if (nRd == 1 || nCd == 1) {
            // one shared line holds all errors: fix each along the orthogonal line
            const bool shared_row = nRd == 1;
            const int one_i = shared_row ? nth_d(R, nR, rc, nrc, 0) : nth_d(C, nC, cc, ncc, 0);
            const double one = shared_row ? Dr[one_i] : Dc[one_i];
            const int *S = shared_row ? C : R;
            const int m = shared_row ? nC : nR;
            const int *s3 = shared_row ? cc : rc;
            const int m3 = shared_row ? ncc : nrc;
            const double *Dm = shared_row ? Dc : Dr;
            double sum = 0.0, sa = 0.0;
            bool nonfin = false;
            for (int a = 0; a < m; a++)
                if (!inset(S[a], s3, m3)) {
                    sum += Dm[S[a]];
                    sa += fabs(Dm[S[a]]);
                    nonfin |= !isfinite(Dm[S[a]]);
                }
            if (nonfin) {
                if (isfinite(one)) return;
            } else if (!d_same(sum, one, 2.0 * tauS + 2.0 * n * EPS * (sa + fabs(one)))) {
                return;
            }
            for (int a = 0; a < m; a++)
                if (!inset(S[a], s3, m3)) {
                    if (shared_row) push(one_i, S[a], 1);  // column formula
                    else push(S[a], one_i, 0);            // row formula
                }
        } else if (nRd == nCd) {
            // distinct rows and columns: pair by value, uniquely in both directions
            for (int a = 0; a < nRd; a++) {
                const int i = nth_d(R, nR, rc, nrc, a);
                int cnt = 0, match = -1;
                for (int b = 0; b < nCd; b++) {
                    const int j = nth_d(C, nC, cc, ncc, b);
                    if (d_same(Dr[i], Dc[j], pair_tol(Dr[i], Dc[j]))) {
                        cnt++;
                        match = j;
                    }
                }
                if (cnt != 1) return;
                int cnt2 = 0;
                for (int a2 = 0; a2 < nRd; a2++) {
                    const int i2 = nth_d(R, nR, rc, nrc, a2);
                    if (d_same(Dr[i2], Dc[match], pair_tol(Dr[i2], Dc[match]))) cnt2++;
                }
                if (cnt2 != 1) return;
                push(i, match, 0);
            }
        } else {
            return;
        }
    }
    for (int q = 0; q < nrc; q++) push(rc[q], -1, 2);
    for (int q = 0; q < ncc; q++) push(-1, cc[q], 3);
    out->nfix = nf;
    out->status = nf > cap ? 3 : 1;
}
cudaError_t ft_decode(const double *Dr, const double *Dc, const double *sums, const double *kap, int n, int mode,
                      const FtCtl *ctl, int *idx, FtFix *fixes, int cap, FtDecOut *out, cudaStream_t s) {
    g_ft_launches++;
    k_decode<<<1, DEC_T, 0, s>>>(Dr, Dc, sums, kap, n, mode, ctl, idx, fixes, cap, out);
    return cudaGetLastError();
}
// the planned fixes (count from the device: blocks past it return), one block per fix
__global__ void k_fix(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode, double *r,
                      int64_t rinc, double *c, int64_t cinc, double *kappa, const FtFix *fixes, double *deltas);
__global__ void k_fix_dev(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode, double *r,
                          int64_t rinc, double *c, int64_t cinc, double *kappa, const FtFix *fixes, double *deltas,
                          const FtDecOut *dec);

// one block per fix: explicit sum excluding the bad element
__device__ void fix_one(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode, double *r,
                        int64_t rinc, double *c, int64_t cinc, double *kappa, const FtFix *fixes, double *deltas);
__global__ void k_fix(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode, double *r,
                      int64_t rinc, double *c, int64_t cinc, double *kappa, const FtFix *fixes, double *deltas) {
    fix_one(Aw, ldw, n, ilo, ihi, cdone, mode, r, rinc, c, cinc, kappa, fixes, deltas);
}
__global__ void k_fix_dev(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode, double *r,
                          int64_t rinc, double *c, int64_t cinc, double *kappa, const FtFix *fixes, double *deltas,
                          const FtDecOut *dec) {
    if (dec->status != 1 || (int)blockIdx.x >= dec->nfix) return;
    fix_one(Aw, ldw, n, ilo, ihi, cdone, mode, r, rinc, c, cinc, kappa, fixes, deltas);
}
__device__ void fix_one(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode, double *r,
                        int64_t rinc, double *c, int64_t cinc, double *kappa, const FtFix *fixes, double *deltas) {
    const FtFix f = fixes[blockIdx.x];
    __shared__ double ws[32];
    double s = 0.0;
    const int i0 = (int)f.i, j0 = (int)f.j;
    if (f.kind == 0 || f.kind == 2 || f.kind == 5) {  // along row i (5: weighted)
        for (int j = threadIdx.x; j < n; j += blockDim.x) {
            if (f.kind == 0 && j == j0) continue;
            bool v = in_v(i0, j, ilo, ihi, cdone);
            if (mode == 0 ? !v : v) s += (f.kind == 5 ? (double)(j + 1) : 1.0) * Aw[i0 + (int64_t)j * ldw];
        }
    } else if (f.kind == 1 || f.kind == 3 || f.kind == 6) {  // along column j (6: weighted)
        for (int i = threadIdx.x; i < n; i += blockDim.x) {
            if (f.kind == 1 && i == i0) continue;
            bool v = in_v(i, j0, ilo, ihi, cdone);
            if (mode == 0 ? !v : v) s += (f.kind == 6 ? (double)(i + 1) : 1.0) * Aw[i + (int64_t)j0 * ldw];
        }
    } else if (f.kind == 7) {  // e^T L w = sum r_w (column n+1)
        for (int i = threadIdx.x; i < n; i += blockDim.x) s += Aw[i + (int64_t)(n + 1) * ldw];
    } else if (f.kind == 8) {  // w^T L e = sum c_w (row n+1)
        for (int j = threadIdx.x; j < n; j += blockDim.x) s += Aw[n + 1 + (int64_t)j * ldw];
    } else {  // kappa = sum r
        for (int i = threadIdx.x; i < n; i += blockDim.x) s += r[(int64_t)i * rinc];
    }
    s = warp_sum(s);
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) t += ws[w];
        double *dst;
        double nv;
        if (f.kind == 0) {
            dst = Aw + i0 + (int64_t)j0 * ldw;
            nv = r[(int64_t)i0 * rinc] - t;
        } else if (f.kind == 1) {
            dst = Aw + i0 + (int64_t)j0 * ldw;
            nv = c[(int64_t)j0 * cinc] - t;
        } else if (f.kind == 2) {
            dst = r + (int64_t)i0 * rinc;
            nv = t;
        } else if (f.kind == 3) {
            dst = c + (int64_t)j0 * cinc;
            nv = t;
        } else if (f.kind == 5) {
            dst = Aw + i0 + (int64_t)(n + 1) * ldw;
            nv = t;
        } else if (f.kind == 6) {
            dst = Aw + n + 1 + (int64_t)j0 * ldw;
            nv = t;
        } else if (f.kind == 7) {
            dst = Aw + n + (int64_t)(n + 1) * ldw;
            nv = t;
        } else if (f.kind == 8) {
            dst = Aw + n + 1 + (int64_t)n * ldw;
            nv = t;
        } else {
            dst = kappa;
            nv = t;
        }
        deltas[blockIdx.x] = nv - *dst;
        *dst = nv;
    }
}
cudaError_t ft_apply_fixes_dev(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode, double *r,
                               int64_t rinc, double *c, int64_t cinc, double *kappa, const FtFix *fixes, int cap,
                               double *deltas, const FtDecOut *dec, cudaStream_t s) {
    g_ft_launches++;
    k_fix_dev<<<cap, 256, 0, s>>>(Aw, ldw, n, ilo, ihi, cdone, mode, r, rinc, c, cinc, kappa, fixes, deltas, dec);
    return cudaGetLastError();
}
cudaError_t ft_apply_fixes(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode, double *r,
                           int64_t rinc, double *c, int64_t cinc, double *kappa, const FtFix *fixes, int nfix,
                           double *deltas, cudaStream_t s) {
    if (nfix <= 0) return cudaSuccess;
    g_ft_launches++;
    k_fix<<<nfix, 256, 0, s>>>(Aw, ldw, n, ilo, ihi, cdone, mode, r, rinc, c, cinc, kappa, fixes, deltas);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// Q formation helpers (ft_dorghr): dense V from the stored reflectors, and T (DLARFT)
// ---------------------------------------------------------------------------
__global__ void k_build_v(const double *Aw, int64_t ldw, double *V, int n, int ihi, int k, int ib, const FtCtl *ctl) {
    if (ctl && ctl->halt) return;
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    int j = blockIdx.y;
    if (i >= n || j >= ib) return;
    int c = k + j;
    double v = 0.0;
    if (i == c + 1) v = 1.0;
    else if (i >= c + 2 && i < ihi) v = Aw[i + (int64_t)c * ldw];
    V[i + (int64_t)j * ldw] = v;
}
// V_chk = e^T V as row n of V (the column-checksum coefficients of the protected Q formation: the
// checksum row c of Q is updated as one more row of the left update, Theorem 1)
__global__ void k_vchk(double *V, int64_t ldw, int n, int k, int ihi, const FtCtl *ctl) {
    if (ctl && ctl->halt) return;
    __shared__ double ws[32];
    const int j = blockIdx.x;
    double sum = 0.0;
    for (int i = k + 1 + threadIdx.x; i < ihi; i += blockDim.x) sum += V[i + (int64_t)j * ldw];
    sum = warp_sum(sum);
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = sum;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) t += ws[w];
        V[n + (int64_t)j * ldw] = t;
    }
}
cudaError_t ft_build_v(const double *Aw, int64_t ldw, double *V, int n, int ihi, int k, int ib, cudaStream_t s,
                       const FtCtl *ctl, int vchk) {
    g_ft_launches++;
    k_build_v<<<dim3((n + 255) / 256, ib), 256, 0, s>>>(Aw, ldw, V, n, ihi, k, ib, ctl);
    if (vchk) {
        g_ft_launches++;
        k_vchk<<<ib, 256, 0, s>>>(V, ldw, n, k, ihi, ctl);
    }
    return cudaGetLastError();
}
// Gram partials of the panel's V over row chunks (DLARFT's V^T V, P:40's compact WY), all SMs:
// block b sums rows [k+1 + b*GR_ROWS, ...) of V(:, a) V(:, bcol) for a < bcol into gpart[b]
#define GR_ROWS 64
__global__ void __launch_bounds__(256) k_gram_part(const double *V, int64_t ldw, int ihi, int k, int ib,
                                                   double *gpart, const FtCtl *ctl) {
    if (ctl && ctl->halt) return;
    __shared__ double Vs[GR_ROWS][FT_NBMAX + 1];
    const int r0 = k + 1 + blockIdx.x * GR_ROWS, r1 = min(ihi, r0 + GR_ROWS), R = r1 - r0;
    for (int x = threadIdx.x; x < GR_ROWS * FT_NBMAX; x += blockDim.x) {
        const int rl = x % GR_ROWS, jj = x / GR_ROWS;
        Vs[rl][jj] = (rl < R && jj < ib) ? V[r0 + rl + (int64_t)jj * ldw] : 0.0;
    }
    __syncthreads();
    double *g = gpart + (int64_t)blockIdx.x * FT_NBMAX * FT_NBMAX;
    for (int pidx = threadIdx.x; pidx < FT_NBMAX * FT_NBMAX; pidx += blockDim.x) {
        const int a = pidx % FT_NBMAX, b = pidx / FT_NBMAX;
        double s0 = 0.0, s1 = 0.0;
        if (a < b && b < ib) {
            int rl = 0;
            for (; rl + 1 < R; rl += 2) {
                s0 += Vs[rl][a] * Vs[rl][b];
                s1 += Vs[rl + 1][a] * Vs[rl + 1][b];
            }
            if (rl < R) s0 += Vs[rl][a] * Vs[rl][b];
        }
        g[pidx] = s0 + s1;
    }
}
// T(0:j, j) = -tau_j T(0:j,0:j) (V(:,0:j)^T v_j), T(j,j) = tau_j  (one block; G = sum of the
// k_gram_part partials in chunk order: deterministic)
__global__ void k_larft(const double *gpart, int nchunk, const double *tau, double *T, int k, int ib,
                        const FtCtl *ctl) {
    if (ctl && ctl->halt) return;
    extern __shared__ double larft_smem[];
    double *G = larft_smem, *Ts = larft_smem + FT_NBMAX * FT_NBMAX, *tmp = Ts + FT_NBMAX * FT_NBMAX;
    for (int pidx = threadIdx.x; pidx < FT_NBMAX * FT_NBMAX; pidx += blockDim.x) {
        double s = 0.0;
        for (int c = 0; c < nchunk; c++) s += __ldcg(gpart + (int64_t)c * FT_NBMAX * FT_NBMAX + pidx);
        G[pidx] = s;
    }
    for (int i = threadIdx.x; i < FT_NBMAX * FT_NBMAX; i += blockDim.x) Ts[i] = 0.0;
    __syncthreads();
    for (int j = 0; j < ib; j++) {
        const double tj = tau[k + j];
        if (threadIdx.x < j) {
            double s = 0.0;
            for (int b = threadIdx.x; b < j; b++) s += Ts[threadIdx.x + b * FT_NBMAX] * G[b + j * FT_NBMAX];
            tmp[threadIdx.x] = -tj * s;
        }
        __syncthreads();
        if (threadIdx.x < j) Ts[threadIdx.x + j * FT_NBMAX] = tmp[threadIdx.x];
        if (threadIdx.x == 0) Ts[j + j * FT_NBMAX] = tj;
        __syncthreads();
    }
    for (int i = threadIdx.x; i < ib * ib; i += blockDim.x) {
        int a = i % ib, b = i / ib;
        T[a + b * FT_NBMAX] = Ts[a + b * FT_NBMAX];
    }
}
cudaError_t ft_larft(const double *V, int64_t ldw, const double *tau, double *T, int n, int ihi, int k, int ib,
                     cudaStream_t s, const FtCtl *ctl, double *gpart) {
    static unsigned attr = 0;
    const unsigned dbit = ft_dev_bit();
    const int smem = (2 * FT_NBMAX * FT_NBMAX + FT_NBMAX) * sizeof(double);
    if (!(attr & dbit)) {
        cudaError_t e = cudaFuncSetAttribute(k_larft, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        attr |= dbit;
    }
    g_ft_launches++;
    const int nchunk = std::max(1, (ihi - k - 1 + GR_ROWS - 1) / GR_ROWS);
    g_ft_launches++;
    k_gram_part<<<nchunk, 256, 0, s>>>(V, ldw, ihi, k, ib, gpart, ctl);
    k_larft<<<1, 512, smem, s>>>(gpart, nchunk, tau, T, k, ib, ctl);
    return cudaGetLastError();
}
__global__ void k_identity(double *Q, int64_t ldq, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    int64_t j = blockIdx.y;
    if (i < n) Q[i + j * ldq] = (i == j) ? 1.0 : 0.0;
}
cudaError_t ft_set_identity(double *Q, int64_t ldq, int n, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    g_ft_launches++;
    k_identity<<<dim3((n + 255) / 256, n), 256, 0, s>>>(Q, ldq, n);
    return cudaGetLastError();
}
// augmented identity of the protected Q formation: Q = I, r = Q e = e (column n), c = e^T Q = e^T
// (row n), kappa = e^T Q e = n (encode, applied to the initial Q)
__global__ void k_identity_aug(double *Q, int64_t ldq, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    int64_t j = blockIdx.y;
    if (i > n) return;
    double v;
    if (i < n && j < n) v = (i == j) ? 1.0 : 0.0;
    else if (i == n && j == n) v = (double)n;
    else v = 1.0;
    Q[i + j * ldq] = v;
}
cudaError_t ft_set_identity_aug(double *Q, int64_t ldq, int n, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    g_ft_launches++;
    k_identity_aug<<<dim3((n + 1 + 255) / 256, n + 1), 256, 0, s>>>(Q, ldq, n);
    return cudaGetLastError();
}
__global__ void k_ctl_norm(FtCtl *ctl, double v) { ctl->normF = v; }
cudaError_t ft_ctl_set_norm(FtCtl *ctl, double v, cudaStream_t s) {
    g_ft_launches++;
    k_ctl_norm<<<1, 1, 0, s>>>(ctl, v);
    return cudaGetLastError();
}

__global__ void k_zero_if_running(double *p, size_t n, const FtCtl *ctl) {
    if (ctl && ctl->halt) return;
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) p[i] = 0.0;
}
cudaError_t ft_zero_if_running(double *p, size_t n, const FtCtl *ctl, cudaStream_t s) {
    g_ft_launches++;
    int blocks = (int)((n + 1023) / 1024);
    if (blocks > 592) blocks = 592;
    k_zero_if_running<<<blocks, 256, 0, s>>>(p, n, ctl);
    return cudaGetLastError();
}
