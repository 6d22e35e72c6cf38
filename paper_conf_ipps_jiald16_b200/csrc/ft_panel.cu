// ft_panel.cu -- persistent DLAHR2 panel kernel (the method's hot spot).
//
// One cooperative launch factorizes one panel of ib columns (DLAHR2, Alg. 2 l.4 /
// Alg. 3 l.5; LAPACK reading R2).  For column c = k + j:
//   (i)   b = A(k+1:n, c) - Y(k+1:n, 0:j) V(c, 0:j)^T                 [row-local]
//   (ii)  b = b - V T^T (V^T b)                                        [grid reduction #1]
//   (iii) DLARFG on (b(c+1), b(c+2:n)) -> beta, tau, v                 [grid reduction #2]
//   (iv)  y = A(k+1:n, c+1:ihi) v   -- the trailing GEMV, ~83% of the  [row-split, no reduction]
//         roofline time of the whole reduction
//   (v)   t = V^T v, Y(:, j) = tau (y - Y t), T(0:j, j) = -tau T t, T(j,j) = tau
// With ABFT the checksum row n rides as one more row of b / Y / V (V_aug(n,:) =
// e^T V = V_chk, Y_aug(n,:) = e^T Y = Y_chk; Alg. 3 l.6-7, readings R7/R8), and the
// first GEMV of the panel also produces row sums of the trailing matrix, so the
// row-checksum discrepancy D_r = r - L e is evaluated BEFORE the panel's output is
// consumed by the updates (verify-before-consume, reading R11/R14).
//
// Layout: rows [rbase, rend) are split into 16-row groups, contiguous per CTA.  Each
// CTA owns its rows for the whole panel (b, Y, V rows); the GEMV reads only its own
// rows of the trailing matrix, so y needs no cross-CTA reduction.  Two grid barriers
// per column; the small reductions are fp64 atomics into triple-buffered accumulators.
#include "ft_common.cuh"
#include "ft_internal.h"

#define PT 512      // threads per CTA
#define NW (PT / 32)
#define VCH 4096    // v chunk staged in shared memory (doubles)

struct PanelSmem {
    double Ts[FT_NBMAX][FT_NBMAX + 1];  // Ts[a][b] = T(a, b)
    double vrow[FT_NBMAX];              // V(c, 0:j) for the current column
    double w[FT_NBMAX], t[FT_NBMAX];
    double bsm[PT];
    double2 redy[PT];
    double2 reds[PT];
    double2 y2[PT / 2];
    double2 rs2[PT / 2];
    // followed (dynamic part) by the CTA's rows of V and Y when they fit: [64][R] each
};

size_t ft_panel_smem_bytes() { return sizeof(PanelSmem); }

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    t = clock64();
    return t;
}
__device__ __forceinline__ unsigned long long gtimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#define PROBE(slot)                                                                   \
    do {                                                                              \
        if (p.dbg && blockIdx.x == 0 && tid == 0 && j < 64)                           \
            p.dbg[j * 16 + (slot)] = gtimer();                                        \
    } while (0)

// sum over the TPR lanes of a row group (TPR is a power of two <= 32, groups are lane-aligned)
__device__ __forceinline__ double group_sum(double v, int tpr) {
#pragma unroll 1
    for (int o = tpr >> 1; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// DLARFG scalars (reading R1), kept out of line: one copy of the division/sqrt/hypot code
struct Refl {
    double tau, beta, scale, vchk;
};
__device__ __noinline__ Refl dlarfg_scalars(double nrm2, double sx, double alpha, bool trivial) {
    Refl r;
    if (nrm2 == 0.0 || trivial) {
        r.tau = 0.0;
        r.beta = alpha;
        r.scale = 1.0;  // H = I, x left untouched (it is zero)
    } else {
        r.beta = -copysign(sqrt(alpha * alpha + nrm2), alpha);  // = -sign(alpha) hypot(alpha, ||x||)
        r.tau = (r.beta - alpha) / r.beta;
        r.scale = 1.0 / (alpha - r.beta);
    }
    r.vchk = 1.0 + r.scale * sx;  // V_chk(j) = e^T v
    return r;
}

template <bool CACHE>
__global__ void __launch_bounds__(PT, 1) k_panel(PanelParams p) {
    if (p.ctl->halt) return;  // uniform for the whole grid (nobody writes halt in this launch)
    extern __shared__ __align__(16) unsigned char smem_raw[];
    PanelSmem &S = *reinterpret_cast<PanelSmem *>(smem_raw);

    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const unsigned P = gridDim.x;
    const int g0 = (int)((long long)blockIdx.x * p.ngroups / P);
    const int g1 = (int)((long long)(blockIdx.x + 1) * p.ngroups / P);
    const int r0 = p.rbase + 16 * g0, r1 = p.rbase + 16 * g1;
    const int R = r1 - r0, R2 = R >> 1;
    const int n = p.n, ihi = p.ihi, k = p.k, ib = p.ib;
    const int64_t ldw = p.ldw;
    double *__restrict__ A = p.A;
    double *__restrict__ V = p.V;
    double *__restrict__ Y = p.Y;
    unsigned epoch = 0;

    // own rows of V and Y: shared memory (write-through to global) when they fit
    constexpr bool cache = CACHE;
    double *Vl = CACHE ? reinterpret_cast<double *>(smem_raw + sizeof(PanelSmem)) : V + r0;
    double *Yl = CACHE ? Vl + (int64_t)FT_NBMAX * R : Y + r0;
    const int64_t ls = CACHE ? R : ldw;  // column stride of Vl / Yl

    // row-group layout for the row-local dots: TPR lanes per row
    int tpr = 32;
    while (tpr > 1 && tpr * R > PT) tpr >>= 1;
    const int rl = tid / tpr, lr = tid % tpr;
    const int row = r0 + rl;
    const bool mine = rl < R;
    const bool datarow = mine && row >= k + 1 && row < ihi;
    const bool chkrow = mine && p.abft && row == n;
    const bool valid = datarow || chkrow;
    const bool leader = mine && lr == 0;

    #pragma unroll 1
    for (int i = tid; i < FT_NBMAX * (FT_NBMAX + 1); i += PT) (&S.Ts[0][0])[i] = 0.0;

    // GEMV thread mapping: row pair rp, column lane cl
    const int ncl = R2 > 0 ? PT / R2 : 0;
    const int rp = R2 > 0 ? tid % R2 : 0;
    const int cl = R2 > 0 ? tid / R2 : 0;
    const bool gemv_on = R2 > 0 && cl < ncl;
    const double2 *__restrict__ A2 = reinterpret_cast<const double2 *>(A + r0);
    const int64_t ldw2 = ldw >> 1;
    const double c_thr = p.ctl->c_thr;
    const double tau_abs = c_thr * (double)n * 2.220446049250313e-16 * p.ctl->normF;
    double acol = valid ? A[row + (int64_t)k * ldw] : 0.0;  // A(row, c) prefetched one column ahead
    __syncthreads();

    for (int j = 0; j < ib; j++) {
        const int c = k + j;
        double *acc = p.acc + (j % 3) * FT_ACC_STRIDE;
        PROBE(0);
        // ---------------- (i) b0 = A(:,c) - Y V(c,:)^T  (row groups, lanes split j') -----
        double b0 = 0.0;
        if (mine) {
            double sacc = 0.0;
            #pragma unroll 1
            for (int jp = lr; jp < j; jp += tpr) sacc += Yl[rl + jp * ls] * S.vrow[jp];
            sacc = group_sum(sacc, tpr);
            b0 = acol - sacc;
        }
        PROBE(9);
        if (leader) S.bsm[rl] = datarow ? b0 : 0.0;
        __syncthreads();
        PROBE(10);
        if (j > 0) {
            // s1 = V^T b0 over data rows (grid reduction #1)
            #pragma unroll 1
            for (int jp = wid; jp < j; jp += NW) {
                double sacc = 0.0;
                #pragma unroll 1
                for (int t = lane; t < R; t += 32) sacc += Vl[t + jp * ls] * S.bsm[t];
                sacc = warp_sum(sacc);
                if (lane == 0 && !(p.dbg_mode & 4)) atomicAdd(acc + jp, sacc);
            }
            PROBE(1);
            if (!(p.dbg_mode & 1)) grid_barrier(p.bar, epoch, P);
            PROBE(2);
            // ---------------- (ii) w = T^T s1 (8 lanes per output) ----------------------
            {
                const int a = tid >> 3, q = tid & 7;
                double sacc = 0.0;
                if (a < j)
                    #pragma unroll 1
                    for (int bb = q; bb <= a; bb += 8) sacc += S.Ts[bb][a] * ldcg(acc + bb);
                sacc += __shfl_xor_sync(0xffffffffu, sacc, 1);
                sacc += __shfl_xor_sync(0xffffffffu, sacc, 2);
                sacc += __shfl_xor_sync(0xffffffffu, sacc, 4);
                if (a < j && q == 0) S.w[a] = sacc;
            }
            PROBE(11);
            __syncthreads();
            PROBE(12);
        }
        double b = b0;
        if (mine && j > 0) {
            double sacc = 0.0;
            #pragma unroll 1
            for (int jp = lr; jp < j; jp += tpr) sacc += Vl[rl + jp * ls] * S.w[jp];
            b = b0 - group_sum(sacc, tpr);
        }
        const bool xrow = datarow && row >= c + 2;
        if (leader) {
            S.bsm[rl] = xrow ? b : 0.0;
            if (xrow) p.bvec[row] = b;
        }
        if (leader && datarow && row == c + 1) acc[2 * FT_NBMAX + 2] = b;  // alpha: a single writer
        __syncthreads();
        // vtb = V(c+2:ihi, :)^T b(c+2:ihi) for jp < j, plus ||x||^2 (jp = j) and sum x (jp = j+1)
#pragma unroll 1
        for (int jp = wid; jp < j + 2; jp += NW) {
            double sacc = 0.0;
#pragma unroll 1
            for (int t = lane; t < R; t += 32) {
                const double bt = S.bsm[t];
                sacc += (jp < j ? Vl[t + jp * ls] : (jp == j ? bt : 1.0)) * bt;
            }
            sacc = warp_sum(sacc);
            if (lane == 0 && !(p.dbg_mode & 4))
                atomicAdd(acc + (jp < j ? FT_NBMAX + jp : 2 * FT_NBMAX + (jp - j)), sacc);
        }
        if (blockIdx.x == 0 && j >= 2) {  // recycle the set used by column j-2
            double *nxt = p.acc + ((j + 1) % 3) * FT_ACC_STRIDE;
            #pragma unroll 1
            for (int i = tid; i < FT_ACC_STRIDE; i += PT) nxt[i] = 0.0;
        }
        PROBE(3);
        if (p.dbg && tid == 0 && j == 5) p.dbg[1024 + blockIdx.x] = gtimer_ns();
        if (!(p.dbg_mode & 1)) grid_barrier(p.bar, epoch, P);
        PROBE(4);
        // ---------------- (iii) DLARFG (reading R1), redundantly in every thread -------
        double vn = 0.0, vt = 0.0;
        if (tid < j) {  // V(c+1, :) (next column's vrow) and V^T b, loaded together with the scalars
            vn = ldcg(V + (c + 1) + (int64_t)tid * ldw);
            vt = ldcg(acc + FT_NBMAX + tid);
        }
        const double alpha = ldcg(acc + 2 * FT_NBMAX + 2);
        const Refl rf = dlarfg_scalars(ldcg(acc + 2 * FT_NBMAX + 0), ldcg(acc + 2 * FT_NBMAX + 1), alpha, c + 2 >= ihi);
        const double tau = rf.tau, beta = rf.beta, scale = rf.scale, vchk = rf.vchk;
        // t = V^T v = V(c+1,:)^T + scale * vtb; V(c+1, :) is also next column's vrow
        if (tid < j) {
            S.t[tid] = vn + scale * vt;
            S.vrow[tid] = vn;
        }
        if (tid == j) S.vrow[j] = 1.0;
        // store V(:, j) and the reduced column c of A for own rows
        if (leader) {
            if (valid) {
                double vv, av;
                if (row == n && p.abft) {
                    vv = vchk;
                    av = (tau != 0.0) ? b - vchk * (alpha - beta) : b;  // left term of reflector j (R7)
                } else if (row <= c) {
                    vv = 0.0;
                    av = b;
                } else if (row == c + 1) {
                    vv = 1.0;
                    av = beta;
                } else {
                    vv = scale * b;
                    av = vv;
                }
                V[row + (int64_t)j * ldw] = vv;
                if (cache) Vl[rl + j * ls] = vv;
                A[row + (int64_t)c * ldw] = av;
            } else if (cache) {
                Vl[rl + j * ls] = 0.0;  // rows outside the panel take no part in the V^T b dots
            }
        }
        // next column's A(row, c+1): issue the load now, consume after the GEMV
        const double acol_next = (valid && j + 1 < ib) ? A[row + (int64_t)(c + 1) * ldw] : 0.0;
        PROBE(5);
        // ---------------- (iv) the trailing GEMV, v staged in shared memory ------------
        const bool vfy = (j == 0) && p.verify;
        const int cend = vfy ? n : ihi;
        double2 ya = make_double2(0.0, 0.0), rs = make_double2(0.0, 0.0);
        if (gemv_on && !(p.dbg_mode & 2)) {
            // v(c+1) = 1, v(q) = scale * b(q) for c+2 <= q < ihi, 0 beyond (verify pass only)
            const double *bv = p.bvec;
            int col = c + 1 + cl;
#pragma unroll 1
            for (; col + 7 * ncl < cend; col += 8 * ncl) {
                double2 a[8];
                double v[8];
#pragma unroll
                for (int u = 0; u < 8; u++) {
                    const int q = col + u * ncl;
                    a[u] = A2[(int64_t)q * ldw2 + rp];
                    v[u] = q < ihi ? ldcg(bv + q) : 0.0;
                }
#pragma unroll
                for (int u = 0; u < 8; u++) {
                    const int q = col + u * ncl;
                    const double vv = q == c + 1 ? 1.0 : scale * v[u];
                    ya.x += a[u].x * vv;
                    ya.y += a[u].y * vv;
                    rs.x += a[u].x;
                    rs.y += a[u].y;
                }
            }
#pragma unroll 1
            for (; col < cend; col += ncl) {
                const double2 a = A2[(int64_t)col * ldw2 + rp];
                const double vv = col == c + 1 ? 1.0 : (col < ihi ? scale * ldcg(bv + col) : 0.0);
                ya.x += a.x * vv;
                ya.y += a.y * vv;
                rs.x += a.x;
                rs.y += a.y;
            }
        }
        PROBE(6);
        if (gemv_on) {
            S.redy[tid] = ya;
            S.reds[tid] = rs;
        }
        __syncthreads();
#pragma unroll 1
        for (int q = wid; q < R2; q += NW) {
            double sx2 = 0.0, sy = 0.0;
#pragma unroll 1
            for (int l = lane; l < ncl; l += 32) {
                const double2 u = S.redy[l * R2 + q];
                sx2 += u.x;
                sy += u.y;
            }
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                sx2 += __shfl_xor_sync(0xffffffffu, sx2, o);
                sy += __shfl_xor_sync(0xffffffffu, sy, o);
            }
            if (lane == 0) S.y2[q] = make_double2(sx2, sy);
        }
        if (vfy)  // row sums for the verify-before-consume check (once per panel)
            for (int q = tid; q < R2; q += PT) {
                double tx = 0.0, ty = 0.0;
                for (int l = 0; l < ncl; l++) {
                    const double2 z = S.reds[l * R2 + q];
                    tx += z.x;
                    ty += z.y;
                }
                S.rs2[q] = make_double2(tx, ty);
            }
        __syncthreads();
        PROBE(7);
        // ---------------- (v) Y(:, j), T(:, j) -------------------------------------
        if (mine) {
            double sacc = 0.0;
            #pragma unroll 1
            for (int jp = lr; jp < j; jp += tpr) sacc += Yl[rl + jp * ls] * S.t[jp];
            sacc = group_sum(sacc, tpr);
            if (leader && valid) {
                const double2 yy2 = S.y2[rl >> 1];
                const double yy = tau * (((rl & 1) ? yy2.y : yy2.x) - sacc);
                Y[row + (int64_t)j * ldw] = yy;
                if (cache) Yl[rl + j * ls] = yy;
            }
        }
        if (vfy && leader && datarow) {
            // D_r(row) = r(row) - sum_{col >= k} L(row, col); columns < k are logical zero here
            const double2 z = S.rs2[rl >> 1];
            const double rsum = b0 + ((rl & 1) ? z.y : z.x);
            const double d = A[row + (int64_t)n * ldw] - rsum;
            if (not_within(d, tau_abs)) {
                atomicAdd(&p.ctl->nflag, 1);
            } else if (tau_abs > 0.0) {
                const double rel = fabs(d) / (tau_abs / c_thr);
                atomicMax(&p.ctl->drift_bits, (unsigned long long)__double_as_longlong(rel));
            }
        }
        {   // T(a, j) = -tau * sum_{b=a}^{j-1} T(a, b) t(b), 8 lanes per output
            const int a = tid >> 3, q = tid & 7;
            double sacc = 0.0;
            if (a < j)
                #pragma unroll 1
                for (int bb = a + q; bb < j; bb += 8) sacc += S.Ts[a][bb] * S.t[bb];
            sacc += __shfl_xor_sync(0xffffffffu, sacc, 1);
            sacc += __shfl_xor_sync(0xffffffffu, sacc, 2);
            sacc += __shfl_xor_sync(0xffffffffu, sacc, 4);
            if (a < j && q == 0) S.Ts[a][j] = -tau * sacc;
            if (tid == 0) S.Ts[j][j] = tau;
        }
        if (blockIdx.x == 0 && tid == 0) {
            p.tau[c] = tau;
            if (p.abft) {
                p.Qc[c] = vchk - 1.0;   // Q column checksum
                p.Qc[n] += vchk - 1.0;  // corner of the Q checksums
            }
        }
        acol = acol_next;
        __syncthreads();
        PROBE(8);
    }
    // Q row checksums of the new Householder vectors (Fig. 5): own data rows
    if (p.abft && leader && datarow) {
        double sacc = 0.0;
        #pragma unroll 1
        for (int jj = 0; jj < ib; jj++)
            if (row >= k + jj + 2) sacc += Vl[rl + jj * ls];
        p.Qr[row] += sacc;
    }
    if (blockIdx.x == 0)
        #pragma unroll 1
        for (int i = tid; i < ib * ib; i += PT) {
            int a = i % ib, bb = i / ib;
            p.T[a + bb * FT_NBMAX] = S.Ts[a][bb];
        }
}

cudaError_t ft_launch_panel(const PanelParams &p, int nsm, cudaStream_t s) {
    static int max_smem = 0;
    if (!max_smem) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        cudaError_t e = cudaFuncSetAttribute(k_panel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem);
        if (e != cudaSuccess) return e;
        e = cudaFuncSetAttribute(k_panel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem);
        if (e != cudaSuccess) return e;
    }
    int grid = nsm < p.ngroups ? nsm : p.ngroups;
    if (grid < 1) grid = 1;
    // rows per CTA (max over CTAs) and whether their V/Y rows fit next to the fixed part
    int gmax = (p.ngroups + grid - 1) / grid;
    int rmax = 16 * gmax;
    if (rmax > PT) return cudaErrorInvalidConfiguration;  // n beyond ~75k rows per GPU
    size_t fixed = sizeof(PanelSmem);
    size_t want = fixed + (size_t)2 * FT_NBMAX * rmax * sizeof(double);
    PanelParams pp = p;
    size_t smem = fixed;
    if (want <= (size_t)max_smem) {
        smem = want;
        pp.smem_rows = rmax;
    } else {
        pp.smem_rows = 0;
    }
    void *args[] = {&pp};
    g_ft_launches++;
    const void *fn = pp.smem_rows > 0 ? (const void *)k_panel<true> : (const void *)k_panel<false>;
    return cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(PT), args, smem, s);
}
