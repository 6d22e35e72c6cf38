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

#define GB_N 64   // strip width
#define GB_M 32   // row tile
#define GT 128    // threads
#define CS_LD (GB_M + 4)

struct RightSmem {
    double Vs[GB_N * FT_KPAD];  // V(cols, :)   [col][j]
    double Ys[GB_M * FT_KPAD];  // sign*Y(rows,:) [row][j]
    double Vt[GB_M * FT_KPAD];  // V(rows, :)   [row][j]  (W operand)
    double Cs[GB_N * CS_LD];    // C tile        [col][row]
};

// load a [GB_M x KT] column-major block (rows r.., columns 0..KT-1 of M, ld) into smem
// as [row][j] (stride FT_KPAD), scaled; zero outside rows [lo, hi) and columns [0, K).
// All loads of a thread are issued before any store (memory-level parallelism).
template <int KT>
__device__ __forceinline__ void load_rows_rowmajor(double *dst, const double *M, int64_t ld, int r, int K, int lo,
                                                   int hi, double scale) {
    constexpr int PER = GB_M * KT / GT;
    double v[PER];
#pragma unroll
    for (int u = 0; u < PER; u++) {
        int i = threadIdx.x + u * GT;
        int m = i % GB_M, jj = i / GB_M;
        int rr = r + m;
        v[u] = (jj < K && rr >= lo && rr < hi) ? M[rr + (int64_t)jj * ld] * scale : 0.0;
    }
#pragma unroll
    for (int u = 0; u < PER; u++) {
        int i = threadIdx.x + u * GT;
        dst[(i % GB_M) * FT_KPAD + i / GB_M] = v[u];
    }
}
// V(cols, 0:KT) for a 64-column strip -> smem [col][j]
template <int KT>
__device__ __forceinline__ void load_strip_rowmajor(double *dst, const double *M, int64_t ld, int c0, int K, int ncols) {
    constexpr int PER = GB_N * KT / GT;
#pragma unroll 8
    for (int u = 0; u < PER; u++) {
        int i = threadIdx.x + u * GT;
        int m = i % GB_N, jj = i / GB_N;
        dst[m * FT_KPAD + jj] = (jj < K && m < ncols) ? M[(c0 + m) + (int64_t)jj * ld] : 0.0;
    }
}
// C tile (GB_M rows x GB_N cols) -> registers (8 double2 per thread) -> smem [col][row];
// only rows m in [mlo, mhi) of the tile are touched in global memory (others read as 0)
__device__ __forceinline__ void load_ctile(double *Cs, const double *A, int64_t lda, int cb, int r, int mlo, int mhi,
                                           int ncols, bool vec_ok) {
    constexpr int PER = GB_N * (GB_M / 2) / GT;
    double2 v[PER];
#pragma unroll
    for (int u = 0; u < PER; u++) {
        int i = threadIdx.x + u * GT;
        int cc = i / (GB_M / 2), m2 = (i % (GB_M / 2)) * 2;
        v[u] = make_double2(0.0, 0.0);
        if (cc < ncols) {
            const double *src = A + (int64_t)(cb + cc) * lda + r + m2;
            if (vec_ok && m2 >= mlo && m2 + 1 < mhi) {
                v[u] = *reinterpret_cast<const double2 *>(src);
            } else {
                if (m2 >= mlo && m2 < mhi) v[u].x = src[0];
                if (m2 + 1 >= mlo && m2 + 1 < mhi) v[u].y = src[1];
            }
        }
    }
#pragma unroll
    for (int u = 0; u < PER; u++) {
        int i = threadIdx.x + u * GT;
        int cc = i / (GB_M / 2), m2 = (i % (GB_M / 2)) * 2;
        *reinterpret_cast<double2 *>(&Cs[cc * CS_LD + m2]) = v[u];
    }
}
__device__ __forceinline__ void store_ctile(const double *Cs, double *A, int64_t lda, int cb, int r, int mlo, int mhi,
                                            int ncols, bool vec_ok) {
    constexpr int PER = GB_N * (GB_M / 2) / GT;
#pragma unroll
    for (int u = 0; u < PER; u++) {
        int i = threadIdx.x + u * GT;
        int cc = i / (GB_M / 2), m2 = (i % (GB_M / 2)) * 2;
        if (cc >= ncols) continue;
        double *dst = A + (int64_t)(cb + cc) * lda + r + m2;
        double2 v = *reinterpret_cast<const double2 *>(&Cs[cc * CS_LD + m2]);
        if (vec_ok && m2 >= mlo && m2 + 1 < mhi) {
            *reinterpret_cast<double2 *>(dst) = v;
        } else {
            if (m2 >= mlo && m2 < mhi) dst[0] = v.x;
            if (m2 + 1 >= mlo && m2 + 1 < mhi) dst[1] = v.y;
        }
    }
}

template <int KT>
__global__ void __launch_bounds__(GT, 2) k_gemm_right(GemmRightParams p) {
    if (p.ctl && p.ctl->halt) return;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    RightSmem &S = *reinterpret_cast<RightSmem *>(smem_raw);
    const int warp = threadIdx.x >> 5;
    const int cb = p.c_lo + blockIdx.x * GB_N;
    const int ncols = min(GB_N, p.c_hi - cb);
    const int K = p.K;
    const bool vec_ok = ((p.lda & 1) == 0) && ((((uintptr_t)p.A) & 15) == 0);
    // row tiles are aligned to absolute multiples of GB_M (16-byte aligned columns)
    const int rbase = (p.r_lo / GB_M) * GB_M;
    const int nrt = (p.r_hi - rbase + GB_M - 1) / GB_M;
    const int t0 = (int)((long long)blockIdx.y * nrt / gridDim.y);
    const int t1 = (int)((long long)(blockIdx.y + 1) * nrt / gridDim.y);

    if (p.do_right) load_strip_rowmajor<KT>(S.Vs, p.V, p.ldw, cb, K, ncols);
    double wacc[4][4][2];
#pragma unroll
    for (int a = 0; a < 4; a++)
#pragma unroll
        for (int b = 0; b < 4; b++) wacc[a][b][0] = wacc[a][b][1] = 0.0;

    for (int tt = t0; tt < t1; tt++) {
        const int r = rbase + tt * GB_M;
        const int lo = max(r, p.r_lo), hi = min(r + GB_M, p.r_hi);
        __syncthreads();
        if (p.do_right) load_rows_rowmajor<KT>(S.Ys, p.Y, p.ldw, r, K, lo, hi, p.sign);
        if (p.do_w) load_rows_rowmajor<KT>(S.Vt, p.V, p.ldw, r, K, max(lo, p.wr_lo), min(hi, p.wr_hi), 1.0);
        load_ctile(S.Cs, p.A, p.lda, cb, r, lo - r, hi - r, ncols, vec_ok);
        __syncthreads();
        if (p.do_right) {
            // warp owns rows 0..31 x cols warp*16 .. +16; rows outside [lo, hi) carry Y = 0
            double acc[4][2][2];
#pragma unroll
            for (int mi = 0; mi < 4; mi++)
#pragma unroll
                for (int ni = 0; ni < 2; ni++)
#pragma unroll
                    for (int v = 0; v < 2; v++)
                        acc[mi][ni][v] = S.Cs[(warp * 16 + frag_col(ni, v)) * CS_LD + frag_row(mi)];
            warp_mma<4, 2, false>(acc, S.Ys, FT_KPAD, S.Vs, FT_KPAD, 0, warp * 16, KT);
            __syncwarp();
#pragma unroll
            for (int mi = 0; mi < 4; mi++)
#pragma unroll
                for (int ni = 0; ni < 2; ni++)
#pragma unroll
                    for (int v = 0; v < 2; v++)
                        S.Cs[(warp * 16 + frag_col(ni, v)) * CS_LD + frag_row(mi)] = acc[mi][ni][v];
            __syncthreads();
            store_ctile(S.Cs, p.A, p.lda, cb, r, lo - r, hi - r, ncols, vec_ok);
        }
        if (p.do_w) {
            // W (KT x 64) += V_tile^T (KT x 32) * C (32 x 64); warp tile 32 x 32
            const int wm0 = (warp >> 1) * 32, wn0 = (warp & 1) * 32;
            if (wm0 < KT) warp_mma<4, 4, true>(wacc, S.Vt, FT_KPAD, S.Cs, CS_LD, wm0, wn0, GB_M);
        }
    }
    if (p.do_w) {
        const int wm0 = (warp >> 1) * 32, wn0 = (warp & 1) * 32;
        double *Wp = p.Wpart + (int64_t)blockIdx.y * p.wsplit_stride;
        if (wm0 < KT) {
#pragma unroll
            for (int mi = 0; mi < 4; mi++)
#pragma unroll
                for (int ni = 0; ni < 4; ni++)
#pragma unroll
                    for (int v = 0; v < 2; v++) {
                        int jj = wm0 + frag_row(mi);
                        int cc = wn0 + frag_col(ni, v);
                        if (jj < K && cc < ncols) Wp[(int64_t)(cb + cc) * FT_NBMAX + jj] = wacc[mi][ni][v];
                    }
        }
    }
}

template <int KT>
static cudaError_t launch_right_kt(const GemmRightParams &p, cudaStream_t s) {
    static bool attr = false;
    size_t smem = sizeof(RightSmem);
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
    return p.K <= 32 ? launch_right_kt<32>(p, s) : launch_right_kt<64>(p, s);
}

// ---------------------------------------------------------------------------
// Left update: A(rows, cols) += sign * V(rows,:) (op(T) W(:, cols))
// ---------------------------------------------------------------------------
struct LeftSmem {
    double Wp[GB_N * FT_KPAD];  // sign*op(T) W [col][j]
    union {
        struct {                // prologue only
            double Ts[FT_NBMAX * FT_NBMAX];
            double Wr[GB_N * FT_KPAD];  // raw W [col][j]
        } pro;
        struct {                // main loop
            double Vt[GB_M * FT_KPAD];
            double Cs[GB_N * CS_LD];
        } main;
    } u;
};

template <int KT>
__global__ void __launch_bounds__(GT, 2) k_gemm_left(GemmLeftParams p) {
    if (p.ctl && p.ctl->halt) return;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    LeftSmem &S = *reinterpret_cast<LeftSmem *>(smem_raw);
    const int warp = threadIdx.x >> 5;
    const int cb = p.c_lo + blockIdx.x * GB_N;
    const int ncols = min(GB_N, p.c_hi - cb);
    const int K = p.K;
    const bool vec_ok = ((p.lda & 1) == 0) && ((((uintptr_t)p.A) & 15) == 0);
    const int rbase = (p.r_lo / GB_M) * GB_M;
    const int nrt = (p.r_hi - rbase + GB_M - 1) / GB_M;
    const int t0 = (int)((long long)blockIdx.y * nrt / gridDim.y);
    const int t1 = (int)((long long)(blockIdx.y + 1) * nrt / gridDim.y);

    for (int i = threadIdx.x; i < K * K; i += blockDim.x) {
        int a = i % K, b = i / K;
        S.u.pro.Ts[a + b * FT_NBMAX] = p.T[a + b * FT_NBMAX];
    }
    for (int i = threadIdx.x; i < GB_N * KT; i += blockDim.x) {
        int jj = i % KT, cc = i / KT;
        double sacc = 0.0;
        if (cc < ncols && jj < K)
            for (int sp = 0; sp < p.nsplit; sp++)
                sacc += p.Wpart[sp * p.wsplit_stride + (int64_t)(cb + cc) * FT_NBMAX + jj];
        S.u.pro.Wr[cc * FT_KPAD + jj] = sacc;
    }
    __syncthreads();
    // Wp(a, col) = sign * sum_b op(T)(a, b) W(b, col);  T upper triangular
    for (int i = threadIdx.x; i < GB_N * KT; i += blockDim.x) {
        int a = i % KT, cc = i / KT;
        double sacc = 0.0;
        if (a < K) {
            if (p.transT) {
                for (int b = 0; b <= a; b++) sacc += S.u.pro.Ts[b + a * FT_NBMAX] * S.u.pro.Wr[cc * FT_KPAD + b];
            } else {
                for (int b = a; b < K; b++) sacc += S.u.pro.Ts[a + b * FT_NBMAX] * S.u.pro.Wr[cc * FT_KPAD + b];
            }
        }
        S.Wp[cc * FT_KPAD + a] = p.sign * sacc;
    }
    for (int tt = t0; tt < t1; tt++) {
        const int r = rbase + tt * GB_M;
        const int lo = max(r, p.r_lo), hi = min(r + GB_M, p.r_hi);
        __syncthreads();
        load_rows_rowmajor<KT>(S.u.main.Vt, p.V, p.ldw, r, K, lo, hi, 1.0);
        load_ctile(S.u.main.Cs, p.A, p.lda, cb, r, lo - r, hi - r, ncols, vec_ok);
        __syncthreads();
        double acc[4][2][2];
#pragma unroll
        for (int mi = 0; mi < 4; mi++)
#pragma unroll
            for (int ni = 0; ni < 2; ni++)
#pragma unroll
                for (int v = 0; v < 2; v++)
                    acc[mi][ni][v] = S.u.main.Cs[(warp * 16 + frag_col(ni, v)) * CS_LD + frag_row(mi)];
        warp_mma<4, 2, false>(acc, S.u.main.Vt, FT_KPAD, S.Wp, FT_KPAD, 0, warp * 16, KT);
        __syncwarp();
#pragma unroll
        for (int mi = 0; mi < 4; mi++)
#pragma unroll
            for (int ni = 0; ni < 2; ni++)
#pragma unroll
                for (int v = 0; v < 2; v++)
                    S.u.main.Cs[(warp * 16 + frag_col(ni, v)) * CS_LD + frag_row(mi)] = acc[mi][ni][v];
        __syncthreads();
        store_ctile(S.u.main.Cs, p.A, p.lda, cb, r, lo - r, hi - r, ncols, vec_ok);
    }
}

template <int KT>
static cudaError_t launch_left_kt(const GemmLeftParams &p, cudaStream_t s) {
    static bool attr = false;
    size_t smem = sizeof(LeftSmem);
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
    g_ft_launches++;
    k_gemm_left<KT><<<dim3(nstrip, ny), GT, smem, s>>>(p);
    return cudaGetLastError();
}
cudaError_t ft_launch_gemm_left(const GemmLeftParams &p, cudaStream_t s) {
    if (p.r_hi <= p.r_lo || p.c_hi <= p.c_lo || p.K <= 0) return cudaSuccess;
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
