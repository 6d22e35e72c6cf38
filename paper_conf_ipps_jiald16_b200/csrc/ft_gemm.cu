// ft_gemm.cu -- FP64 tensor-core (DMMA) block-reflector updates on the augmented matrix.
//
// Right update (Alg. 3 l.8/l.10; Fig. 4c-d):  A_aug(rows, cols) -= Y_aug V_aug(cols,:)^T
// fused with W = V^T A_new (the first half of the left update, DLARFB 'L','T' P:42/P:56 l.8),
// and the left update (Alg. 3 l.11, Fig. 4e):         A_aug(rows, cols) -= V_aug (T^T W).
// Row n of Y_aug/V_aug is Y_chk / V_chk and column n of A_aug is the row checksum r, row n
// the column checksum c -- so Theorem 1 is carried by the same tiles.
// Rollback (reverse computation, Alg. 3 l.14) is the same kernels with sign +1.
//
// Tiling: a CTA owns a 64-column strip and a contiguous row range; it walks the rows in
// 32-row tiles staged in shared memory (coalesced 16-byte loads), the MMA is
// mma.sync.m8n8k4.f64 (SASS DMMA) on 4 warps.  W partials are written per row split and
// reduced (with T^T) in the prologue of the left-update kernel, so both passes are
// deterministic.
#include "ft_common.cuh"
#include "ft_internal.h"

#define GB_N 64   // strip width (columns of the updated matrix per CTA)
#define GB_M 32   // row tile
#define GT 128    // threads (4 warps)
#define TS (GB_M + 4)   // smem stride of row-indexed tiles (36 = 4 mod 16: conflict-free)

template <int KT>
struct RightSmemT {
    double Vs[KT][GB_N + 4];  // V(cols, j) as [j][col]: B operand of the right update (k-major)
    struct Stage {
        double Cs[GB_N][TS];  // C tile [col][row] (column-major, as in HBM)
        double Ys[KT][TS];    // Y(rows, j) as [j][row]
        double Vt[KT][TS];    // V(rows, j) as [j][row]: A operand of W = V^T C
    } st[2];
};

// stage loaders (cp.async 16 B chunks; rows >= hi of the tile are zero-filled, never read)
__device__ __forceinline__ void issue_ctile(double (*Cs)[TS], const double *A, int64_t lda, int cb, int r, int hi,
                                            int ncols) {
    for (int q = threadIdx.x; q < GB_N * (GB_M / 2); q += GT) {
        int cc = q / (GB_M / 2), m2 = (q % (GB_M / 2)) * 2;
        int rows_left = hi - (r + m2);
        int bytes = (cc < ncols) ? (rows_left >= 2 ? 16 : (rows_left == 1 ? 8 : 0)) : 0;
        const double *src = bytes ? A + (int64_t)(cb + cc) * lda + r + m2 : A;
        cp_async16(&Cs[cc][m2], src, bytes);
    }
}
template <int KT>
__device__ __forceinline__ void issue_jtile(double (*T)[TS], const double *M, int64_t ld, int r, int K) {
    for (int q = threadIdx.x; q < KT * (GB_M / 2); q += GT) {
        int jj = q / (GB_M / 2), m2 = (q % (GB_M / 2)) * 2;
        int bytes = jj < K ? 16 : 0;
        const double *src = bytes ? M + (int64_t)jj * ld + r + m2 : M;
        cp_async16(&T[jj][m2], src, bytes);
    }
}
// zero rows of a [KT][TS] tile outside [lo, hi) (tile rows r .. r+GB_M)
template <int KT>
__device__ __forceinline__ void mask_jtile(double (*T)[TS], int r, int lo, int hi) {
    if (r >= lo && r + GB_M <= hi) return;
    for (int q = threadIdx.x; q < KT * GB_M; q += GT) {
        int jj = q / GB_M, m = q % GB_M;
        if (r + m < lo || r + m >= hi) T[jj][m] = 0.0;
    }
}
__device__ __forceinline__ void store_ctile2(double (*Cs)[TS], double *A, int64_t lda, int cb, int r, int lo, int hi,
                                             int ncols) {
    for (int q = threadIdx.x; q < GB_N * (GB_M / 2); q += GT) {
        int cc = q / (GB_M / 2), m2 = (q % (GB_M / 2)) * 2;
        if (cc >= ncols) continue;
        int row = r + m2;
        double *dst = A + (int64_t)(cb + cc) * lda + row;
        double2 v = *reinterpret_cast<const double2 *>(&Cs[cc][m2]);
        if (row >= lo && row + 1 < hi) {
            *reinterpret_cast<double2 *>(dst) = v;
        } else {
            if (row >= lo && row < hi) dst[0] = v.x;
            if (row + 1 >= lo && row + 1 < hi) dst[1] = v.y;
        }
    }
}

// ---------------------------------------------------------------------------
// Right update A(rows, cols) += sign * Y V(cols,:)^T, fused W = V(wrows,:)^T A_new
// ---------------------------------------------------------------------------
template <int KT>
__global__ void __launch_bounds__(GT) k_gemm_right(GemmRightParams p) {
    if (p.ctl && p.ctl->halt) return;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    RightSmemT<KT> &S = *reinterpret_cast<RightSmemT<KT> *>(smem_raw);
    const int warp = threadIdx.x >> 5;
    const int cb = p.c_lo + blockIdx.x * GB_N;
    const int ncols = min(GB_N, p.c_hi - cb);
    const int K = p.K;
    const double sg = p.sign;
    const int rbase = (p.r_lo / GB_M) * GB_M;  // 256-byte aligned tiles
    const int nrt = (p.r_hi - rbase + GB_M - 1) / GB_M;
    const int t0 = (int)((long long)blockIdx.y * nrt / gridDim.y);
    const int t1 = (int)((long long)(blockIdx.y + 1) * nrt / gridDim.y);

    // V(cols, :) once per CTA, [j][col]
    if (p.do_right) {
        constexpr int PER = KT * GB_N / GT;
        double tmp[PER];
#pragma unroll
        for (int u = 0; u < PER; u++) {
            int q = threadIdx.x + u * GT, jj = q / GB_N, cc = q % GB_N;
            tmp[u] = (jj < K && cc < ncols) ? __ldg(p.V + (cb + cc) + (int64_t)jj * p.ldw) : 0.0;
        }
#pragma unroll
        for (int u = 0; u < PER; u++) {
            int q = threadIdx.x + u * GT;
            S.Vs[q / GB_N][q % GB_N] = tmp[u];
        }
    }
    constexpr int WMI = 4, WNI = KT == 64 ? 4 : 2;  // W warp tile: 32 j x (8*WNI) cols
    double wacc[WMI][WNI][2];
#pragma unroll
    for (int a = 0; a < WMI; a++)
#pragma unroll
        for (int b = 0; b < WNI; b++) wacc[a][b][0] = wacc[a][b][1] = 0.0;
    const int wm0 = KT == 64 ? (warp >> 1) * 32 : 0;
    const int wn0 = KT == 64 ? (warp & 1) * 32 : warp * 16;

    auto issue = [&](int tt, int s) {
        const int r = rbase + tt * GB_M;
        const int hi = min(r + GB_M, p.r_hi);
        issue_ctile(S.st[s].Cs, p.A, p.lda, cb, r, hi, ncols);
        if (p.do_right) issue_jtile<KT>(S.st[s].Ys, p.Y, p.ldw, r, K);
        if (p.do_w) issue_jtile<KT>(S.st[s].Vt, p.V, p.ldw, r, K);
        cp_async_commit();
    };
    if (t0 < t1) issue(t0, 0);
    for (int tt = t0; tt < t1; tt++) {
        const int s = (tt - t0) & 1;
        const int r = rbase + tt * GB_M;
        const int lo = max(r, p.r_lo), hi = min(r + GB_M, p.r_hi);
        if (tt + 1 < t1) {
            issue(tt + 1, s ^ 1);
            cp_async_wait<1>();
        } else {
            cp_async_wait<0>();
        }
        __syncthreads();
        auto &St = S.st[s];
        if (p.do_w) {
            mask_jtile<KT>(St.Vt, r, max(lo, p.wr_lo), min(hi, p.wr_hi));
        }
        if (p.do_right) {
            // C' = C + sg * Y V^T:  acc = sg*C ; acc += Y V^T ; C' = sg*acc
            double acc[4][2][2];
#pragma unroll
            for (int mi = 0; mi < 4; mi++)
#pragma unroll
                for (int ni = 0; ni < 2; ni++)
#pragma unroll
                    for (int v = 0; v < 2; v++)
                        acc[mi][ni][v] = sg * St.Cs[warp * 16 + frag_col(ni, v)][frag_row(mi)];
            warp_mma2<4, 2, true, true>(acc, &St.Ys[0][0], TS, &S.Vs[0][0], GB_N + 4, 0, warp * 16, KT);
#pragma unroll
            for (int mi = 0; mi < 4; mi++)
#pragma unroll
                for (int ni = 0; ni < 2; ni++)
#pragma unroll
                    for (int v = 0; v < 2; v++)
                        St.Cs[warp * 16 + frag_col(ni, v)][frag_row(mi)] = sg * acc[mi][ni][v];
            __syncthreads();
            store_ctile2(St.Cs, p.A, p.lda, cb, r, lo, hi, ncols);
        } else if (p.do_w) {
            __syncthreads();
        }
        if (p.do_w) {
            // rows outside [lo, hi) of the C tile are stale/zero, Vt is zero there
            warp_mma2<WMI, WNI, false, false>(wacc, &St.Vt[0][0], TS, &St.Cs[0][0], TS, wm0, wn0, GB_M);
        }
        __syncthreads();
    }
    if (p.do_w) {
        // row splits of a strip accumulate into one W (fp64 RED at L2; W zeroed by the host)
        double *Wp = p.Wpart;
#pragma unroll
        for (int mi = 0; mi < WMI; mi++)
#pragma unroll
            for (int ni = 0; ni < WNI; ni++)
#pragma unroll
                for (int v = 0; v < 2; v++) {
                    int jj = wm0 + frag_row(mi);
                    int cc = wn0 + frag_col(ni, v);
                    if (jj < K && cc < ncols) {
                        double *dst = Wp + (int64_t)(cb + cc) * FT_NBMAX + jj;
                        if (gridDim.y == 1) *dst = wacc[mi][ni][v];
                        else atomicAdd(dst, wacc[mi][ni][v]);
                    }
                }
    }
}

template <int KT>
static cudaError_t launch_right_kt(const GemmRightParams &p, cudaStream_t s) {
    static bool attr = false;
    size_t smem = sizeof(RightSmemT<KT>);
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(k_gemm_right<KT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    int nstrip = (p.c_hi - p.c_lo + GB_N - 1) / GB_N;
    int ny = p.nsplit > 0 ? p.nsplit : 1;
    g_ft_launches++;
    k_gemm_right<KT><<<dim3(nstrip, ny), GT, smem, s>>>(p);
    return cudaGetLastError();
}
cudaError_t ft_launch_gemm_right(const GemmRightParams &p, cudaStream_t s) {
    if (p.r_hi <= p.r_lo || p.c_hi <= p.c_lo || p.K <= 0) return cudaSuccess;
    const bool aligned = (p.lda % 2 == 0) && ((((uintptr_t)p.A) & 15) == 0) && (p.ldw % 2 == 0) &&
                         ((((uintptr_t)p.V) & 15) == 0) && (!p.do_right || ((((uintptr_t)p.Y) & 15) == 0));
    if (!aligned) return cudaErrorInvalidValue;  // the library only passes 16-byte aligned operands
    return p.K <= 32 ? launch_right_kt<32>(p, s) : launch_right_kt<64>(p, s);
}

// ---------------------------------------------------------------------------
// Left update: A(rows, cols) += sign * V(rows,:) (op(T) W(:, cols))
// ---------------------------------------------------------------------------
template <int KT>
struct LeftSmemT {
    double Wp[GB_N][KT + 4];  // op(T) W as [col][j]: B operand (n-major)
    struct {
        double Cs[GB_N][TS];
        double Vt[KT][TS];
    } st[2];
};

// W'(col, a) = sum_b op(T)(a, b) W(b, col), T upper triangular; W, W' stored [col][64]
__global__ void k_wprep(const double *__restrict__ W, const double *__restrict__ T, double *__restrict__ Wt,
                        int c_lo, int c_hi, int K, int transT, const FtCtl *ctl) {
    if (ctl && ctl->halt) return;
    __shared__ double Ts[FT_NBMAX][FT_NBMAX + 1];
    for (int i = threadIdx.x; i < K * K; i += blockDim.x) {
        int a = i % K, b = i / K;
        Ts[a][b] = T[a + b * FT_NBMAX];
    }
    __syncthreads();
    const int a = threadIdx.x % FT_NBMAX;
    const int col = c_lo + blockIdx.x * (blockDim.x / FT_NBMAX) + threadIdx.x / FT_NBMAX;
    if (col >= c_hi || a >= K) return;
    const double *w = W + (int64_t)col * FT_NBMAX;
    double s0 = 0.0, s1 = 0.0;
    if (transT) {
        int b = 0;
        for (; b + 1 <= a; b += 2) {
            s0 += Ts[b][a] * w[b];
            s1 += Ts[b + 1][a] * w[b + 1];
        }
        if (b <= a) s0 += Ts[b][a] * w[b];
    } else {
        int b = a;
        for (; b + 1 < K; b += 2) {
            s0 += Ts[a][b] * w[b];
            s1 += Ts[a][b + 1] * w[b + 1];
        }
        if (b < K) s0 += Ts[a][b] * w[b];
    }
    Wt[(int64_t)col * FT_NBMAX + a] = s0 + s1;
}

template <int KT>
__global__ void __launch_bounds__(GT) k_gemm_left(GemmLeftParams p) {
    if (p.ctl && p.ctl->halt) return;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    LeftSmemT<KT> &S = *reinterpret_cast<LeftSmemT<KT> *>(smem_raw);
    const int warp = threadIdx.x >> 5;
    const int cb = p.c_lo + blockIdx.x * GB_N;
    const int ncols = min(GB_N, p.c_hi - cb);
    const int K = p.K;
    const double sg = p.sign;
    const int rbase = (p.r_lo / GB_M) * GB_M;
    const int nrt = (p.r_hi - rbase + GB_M - 1) / GB_M;
    const int t0 = (int)((long long)blockIdx.y * nrt / gridDim.y);
    const int t1 = (int)((long long)(blockIdx.y + 1) * nrt / gridDim.y);

    // W' for this strip: [col][j] rows of 64 doubles in HBM -> [col][KT+4] in smem
    for (int q = threadIdx.x; q < GB_N * (KT / 2); q += GT) {
        int cc = q / (KT / 2), j2 = (q % (KT / 2)) * 2;
        int bytes = cc < ncols ? 16 : 0;
        const double *src = bytes ? p.Wpart + (int64_t)(cb + cc) * FT_NBMAX + j2 : p.Wpart;
        cp_async16(&S.Wp[cc][j2], src, bytes);
    }
    auto issue = [&](int tt, int s) {
        const int r = rbase + tt * GB_M;
        const int hi = min(r + GB_M, p.r_hi);
        issue_ctile(S.st[s].Cs, p.A, p.lda, cb, r, hi, ncols);
        issue_jtile<KT>(S.st[s].Vt, p.V, p.ldw, r, K);
        cp_async_commit();
    };
    if (t0 < t1) issue(t0, 0);
    else cp_async_commit();
    for (int tt = t0; tt < t1; tt++) {
        const int s = (tt - t0) & 1;
        const int r = rbase + tt * GB_M;
        const int lo = max(r, p.r_lo), hi = min(r + GB_M, p.r_hi);
        if (tt + 1 < t1) {
            issue(tt + 1, s ^ 1);
            cp_async_wait<1>();
        } else {
            cp_async_wait<0>();
        }
        __syncthreads();
        auto &St = S.st[s];
        double acc[4][2][2];
#pragma unroll
        for (int mi = 0; mi < 4; mi++)
#pragma unroll
            for (int ni = 0; ni < 2; ni++)
#pragma unroll
                for (int v = 0; v < 2; v++) acc[mi][ni][v] = sg * St.Cs[warp * 16 + frag_col(ni, v)][frag_row(mi)];
        warp_mma2<4, 2, true, false>(acc, &St.Vt[0][0], TS, &S.Wp[0][0], KT + 4, 0, warp * 16, KT);
#pragma unroll
        for (int mi = 0; mi < 4; mi++)
#pragma unroll
            for (int ni = 0; ni < 2; ni++)
#pragma unroll
                for (int v = 0; v < 2; v++) St.Cs[warp * 16 + frag_col(ni, v)][frag_row(mi)] = sg * acc[mi][ni][v];
        __syncthreads();
        store_ctile2(St.Cs, p.A, p.lda, cb, r, lo, hi, ncols);
        __syncthreads();
    }
}

template <int KT>
static cudaError_t launch_left_kt(const GemmLeftParams &p, cudaStream_t s) {
    static bool attr = false;
    size_t smem = sizeof(LeftSmemT<KT>);
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(k_gemm_left<KT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    int nstrip = (p.c_hi - p.c_lo + GB_N - 1) / GB_N;
    int nrt = (p.r_hi - (p.r_lo / GB_M) * GB_M + GB_M - 1) / GB_M;
    int ny = (2 * 148 + nstrip - 1) / nstrip;
    if (ny > nrt / 2) ny = nrt / 2;
    if (ny < 1) ny = 1;
    g_ft_launches += 2;
    const int per = GT / FT_NBMAX;  // columns per k_wprep block
    k_wprep<<<(p.c_hi - p.c_lo + per - 1) / per, GT, 0, s>>>(p.Wpart, p.T, p.Wt, p.c_lo, p.c_hi, p.K, p.transT,
                                                              p.ctl);
    GemmLeftParams q = p;
    q.Wpart = p.Wt;  // the main kernel reads W' = op(T) W
    k_gemm_left<KT><<<dim3(nstrip, ny), GT, smem, s>>>(q);
    return cudaGetLastError();
}
cudaError_t ft_launch_gemm_left(const GemmLeftParams &p, cudaStream_t s) {
    if (p.r_hi <= p.r_lo || p.c_hi <= p.c_lo || p.K <= 0) return cudaSuccess;
    const bool aligned = (p.lda % 2 == 0) && ((((uintptr_t)p.A) & 15) == 0) && (p.ldw % 2 == 0) &&
                         ((((uintptr_t)p.V) & 15) == 0);
    if (!aligned) return cudaErrorInvalidValue;
    return p.K <= 32 ? launch_left_kt<32>(p, s) : launch_left_kt<64>(p, s);
}

// ---------------------------------------------------------------------------
// Y_top (DLAHR2's final step): Y(0:k+1, :) = A(0:k+1, k+1:ihi) V(k+1:ihi, :) T,
// split over the long inner dimension; the same pass sums A's rows for the
// verify-before-consume check of the rows above the panel (area 1).
// ---------------------------------------------------------------------------
#define YT_M 64
#define YT_K 32
struct YtopSmem {
    double As[YT_K * (YT_M + 4)];        // A tile [col][row]
    double Vs[FT_NBMAX * (YT_K + 4)];    // V [j][col]
    double rsum[YT_M];
};

__global__ void __launch_bounds__(GT) k_ytop_partial(YtopParams p) {
    if (p.ctl->halt) return;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    YtopSmem &S = *reinterpret_cast<YtopSmem *>(smem_raw);
    const int warp = threadIdx.x >> 5;
    const int m_lo = blockIdx.x * YT_M;
    const int mrows = min(YT_M, p.k + 1 - m_lo);
    const int K0 = p.k + 1, K1 = p.ihi;  // inner range
    const int nkt = (K1 - K0 + YT_K - 1) / YT_K;
    const int kt0 = (int)((long long)blockIdx.y * nkt / gridDim.y);
    const int kt1 = (int)((long long)(blockIdx.y + 1) * nkt / gridDim.y);
    const int ib = p.ib;
    double acc[2][8][2];
#pragma unroll
    for (int a = 0; a < 2; a++)
#pragma unroll
        for (int b = 0; b < 8; b++) acc[a][b][0] = acc[a][b][1] = 0.0;
    double rs = 0.0;
    for (int kt = kt0; kt < kt1; kt++) {
        const int kc = K0 + kt * YT_K;
        const int nk = min(YT_K, K1 - kc);
        __syncthreads();
        for (int i = threadIdx.x; i < YT_K * YT_M; i += blockDim.x) {
            int m = i % YT_M, kk = i / YT_M;
            double v = 0.0;
            if (m < mrows && kk < nk) v = p.A[(m_lo + m) + (int64_t)(kc + kk) * p.ldw];
            S.As[kk * (YT_M + 4) + m] = v;
        }
        for (int i = threadIdx.x; i < FT_NBMAX * YT_K; i += blockDim.x) {
            int kk = i % YT_K, jj = i / YT_K;
            double v = 0.0;
            if (jj < ib && kk < nk) v = p.V[(kc + kk) + (int64_t)jj * p.ldw];
            S.Vs[jj * (YT_K + 4) + kk] = v;
        }
        __syncthreads();
        if (p.verify && threadIdx.x < YT_M)
            for (int kk = 0; kk < nk; kk++) rs += S.As[kk * (YT_M + 4) + threadIdx.x];
        // warp tile: rows warp*16..+16, cols 0..63 (MI=2, NI=8)
        warp_mma<2, 8, true>(acc, S.As, YT_M + 4, S.Vs, YT_K + 4, warp * 16, 0, YT_K);
    }
    double *yp = p.ypart + (int64_t)blockIdx.y * (int64_t)(p.k + 1) * FT_NBMAX;
#pragma unroll
    for (int mi = 0; mi < 2; mi++)
#pragma unroll
        for (int ni = 0; ni < 8; ni++)
#pragma unroll
            for (int v = 0; v < 2; v++) {
                int m = warp * 16 + frag_row(mi), jj = frag_col(ni, v);
                if (m < mrows && jj < ib) yp[(int64_t)(m_lo + m) * FT_NBMAX + jj] = acc[mi][ni][v];
            }
    if (p.verify && threadIdx.x < mrows) p.rowpart[(int64_t)blockIdx.y * (p.k + 1) + m_lo + threadIdx.x] = rs;
}

// Y_top rows: sum the split partials, multiply by T; row-sum verify of area 1.
// Block = 16 rows x 64 columns of Y.
#define YF_R 16
__global__ void __launch_bounds__(YF_R * 64) k_ytop_finalize(YtopParams p) {
    if (p.ctl->halt) return;
    __shared__ double Ts[FT_NBMAX * FT_NBMAX];
    __shared__ double y0[YF_R][FT_NBMAX + 1];
    const int jb = threadIdx.x & 63, rl = threadIdx.x >> 6;
    const int row = blockIdx.x * YF_R + rl;
    const int ib = p.ib;
    for (int i = threadIdx.x; i < ib * ib; i += blockDim.x) {
        int a = i % ib, b = i / ib;
        Ts[a + b * FT_NBMAX] = p.T[a + b * FT_NBMAX];
    }
    double acc = 0.0;
    if (row <= p.k && jb < ib)
        for (int sp = 0; sp < p.nsplit; sp++)
            acc += p.ypart[(int64_t)sp * (p.k + 1) * FT_NBMAX + (int64_t)row * FT_NBMAX + jb];
    y0[rl][jb] = acc;
    __syncthreads();
    if (row > p.k) return;
    if (jb < ib) {
        double s = 0.0;
        for (int b = 0; b <= jb; b++) s += y0[rl][b] * Ts[b + jb * FT_NBMAX];
        p.Y[row + (int64_t)jb * p.ldw] = s;
    }
    if (p.verify && jb == 0) {
        double rsum = 0.0;
        for (int sp = 0; sp < p.nsplit; sp++) rsum += p.rowpart[(int64_t)sp * (p.k + 1) + row];
        rsum += p.A[row + (int64_t)p.k * p.ldw];
        for (int col = p.ihi; col < p.n; col++) rsum += p.A[row + (int64_t)col * p.ldw];
        double d = p.A[row + (int64_t)p.n * p.ldw] - p.Fr[row] - rsum;
        double tau_abs = p.ctl->c_thr * (double)p.n * 2.220446049250313e-16 * p.ctl->normF;
        if (not_within(d, tau_abs)) atomicAdd(&p.ctl->nflag, 1);
    }
}

cudaError_t ft_launch_ytop(const YtopParams &p, cudaStream_t s) {
    static bool attr = false;
    size_t smem = sizeof(YtopSmem);
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(k_ytop_partial, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    int nm = (p.k + 1 + YT_M - 1) / YT_M;
    g_ft_launches += 2;
    k_ytop_partial<<<dim3(nm, p.nsplit), GT, smem, s>>>(p);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    k_ytop_finalize<<<(p.k + 1 + YF_R - 1) / YF_R, YF_R * 64, 0, s>>>(p);
    return cudaGetLastError();
}
