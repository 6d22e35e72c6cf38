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
#define VCH 4096    // v chunk staged in shared memory (doubles)

struct PanelSmem {
    double Ts[FT_NBMAX * FT_NBMAX];  // T, column-major (Ts[a + b*64] = T(a,b))
    double vrow[FT_NBMAX], s1[FT_NBMAX], w[FT_NBMAX], t[FT_NBMAX], vtb[FT_NBMAX];
    double vch[VCH];
    double bsm[PT];
    double2 redy[PT];
    double2 reds[PT];
    double2 y2[PT / 2];
    double2 rs2[PT / 2];
    double wred[PT / 32][4];
    double scal[8];
    // followed (dynamic part) by the CTA's rows of V and Y when they fit: [64][R] each
};

size_t ft_panel_smem_bytes() { return sizeof(PanelSmem); }

__device__ __forceinline__ void block_sum3(PanelSmem &S, double &a, double &b, double &c) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    a = warp_sum(a);
    b = warp_sum(b);
    c = warp_sum(c);
    if (lane == 0) {
        S.wred[wid][0] = a;
        S.wred[wid][1] = b;
        S.wred[wid][2] = c;
    }
    __syncthreads();
    if (wid == 0) {
        a = lane < nw ? S.wred[lane][0] : 0.0;
        b = lane < nw ? S.wred[lane][1] : 0.0;
        c = lane < nw ? S.wred[lane][2] : 0.0;
        a = warp_sum(a);
        b = warp_sum(b);
        c = warp_sum(c);
    }
    __syncthreads();
}

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#define PROBE(slot)                                                                   \
    do {                                                                              \
        if (p.dbg && blockIdx.x == 0 && tid == 0 && j < 64)                           \
            p.dbg[j * 16 + (slot)] = gtimer();                                        \
    } while (0)

__global__ void __launch_bounds__(PT, 1) k_panel(PanelParams p) {
    if (p.ctl->halt) return;  // uniform for the whole grid (nobody writes halt in this launch)
    extern __shared__ __align__(16) unsigned char smem_raw[];
    PanelSmem &S = *reinterpret_cast<PanelSmem *>(smem_raw);

    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, nw = blockDim.x >> 5;
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
    const bool cache = p.smem_rows >= R;
    double *Vl = cache ? reinterpret_cast<double *>(smem_raw + sizeof(PanelSmem)) : V + r0;
    double *Yl = cache ? Vl + (int64_t)FT_NBMAX * R : Y + r0;
    const int64_t ls = cache ? R : ldw;  // column stride of Vl / Yl

    const int row = r0 + tid;
    const bool mine = tid < R;
    const bool datarow = mine && row >= k + 1 && row < ihi;
    const bool chkrow = mine && p.abft && row == n;
    const bool valid = datarow || chkrow;

    for (int i = tid; i < FT_NBMAX * FT_NBMAX; i += blockDim.x) S.Ts[i] = 0.0;

    // GEMV thread mapping: row pair rp, column lane cl
    const int ncl = R2 > 0 ? (int)blockDim.x / R2 : 0;
    const int rp = R2 > 0 ? tid % R2 : 0;
    const int cl = R2 > 0 ? tid / R2 : 0;
    const bool gemv_on = R2 > 0 && cl < ncl;
    const double2 *__restrict__ A2 = reinterpret_cast<const double2 *>(A + r0);
    const int64_t ldw2 = ldw >> 1;
    // the panel columns of this CTA's rows stay in registers (one per thread)
    const double tau_abs = p.ctl->c_thr * (double)n * 2.220446049250313e-16 * p.ctl->normF;
    __syncthreads();

    for (int j = 0; j < ib; j++) {
        const int c = k + j;
        double *acc = p.acc + (j % 3) * FT_ACC_STRIDE;
        PROBE(0);
        // ---------------- (i) b0 = A(:,c) - Y V(c,:)^T  ------------------------------
        if (tid < j) S.vrow[tid] = (tid == j - 1) ? 1.0 : ldcg(V + c + (int64_t)tid * ldw);
        __syncthreads();
        double b0 = 0.0;
        if (valid) {
            b0 = A[row + (int64_t)c * ldw];
            for (int jp = 0; jp < j; jp++) b0 -= Yl[tid + jp * ls] * S.vrow[jp];
        }
        S.bsm[tid] = datarow ? b0 : 0.0;
        __syncthreads();
        if (j > 0) {
            // s1 = V^T b0 over data rows (grid reduction #1)
            for (int jp = wid; jp < j; jp += nw) {
                double sacc = 0.0;
                for (int t = lane; t < R; t += 32) sacc += Vl[t + jp * ls] * S.bsm[t];  // bsm = 0 off data rows
                sacc = warp_sum(sacc);
                if (lane == 0) atomicAdd(acc + jp, sacc);
            }
            PROBE(1);
            grid_barrier(p.bar, epoch, P);
            PROBE(2);
            // ---------------- (ii) w = T^T s1 ; b = b0 - V_aug w ----------------------
            if (tid < j) S.s1[tid] = ldcg(acc + tid);
            __syncthreads();
            if (tid < j) {
                double sacc = 0.0;
                for (int bb = 0; bb <= tid; bb++) sacc += S.Ts[bb + tid * FT_NBMAX] * S.s1[bb];
                S.w[tid] = sacc;
            }
            __syncthreads();
        }
        double b = b0;
        if (valid)
            for (int jp = 0; jp < j; jp++) b -= Vl[tid + jp * ls] * S.w[jp];
        const bool xrow = datarow && row >= c + 2;
        if (xrow) p.bvec[row] = b;
        S.bsm[tid] = xrow ? b : 0.0;
        {
            double a1 = xrow ? b * b : 0.0, a2 = xrow ? b : 0.0, a3 = (datarow && row == c + 1) ? b : 0.0;
            block_sum3(S, a1, a2, a3);  // includes __syncthreads
            if (tid == 0) {
                atomicAdd(acc + 2 * FT_NBMAX + 0, a1);
                atomicAdd(acc + 2 * FT_NBMAX + 1, a2);
                atomicAdd(acc + 2 * FT_NBMAX + 2, a3);
            }
        }
        for (int jp = wid; jp < j; jp += nw) {  // vtb = V(c+2:ihi, :)^T b(c+2:ihi)
            double sacc = 0.0;
            for (int t = lane; t < R; t += 32) sacc += Vl[t + jp * ls] * S.bsm[t];
            sacc = warp_sum(sacc);
            if (lane == 0) atomicAdd(acc + FT_NBMAX + jp, sacc);
        }
        if (blockIdx.x == 0 && j >= 2) {  // recycle the set used by column j-2
            double *nxt = p.acc + ((j + 1) % 3) * FT_ACC_STRIDE;
            for (int i = tid; i < FT_ACC_STRIDE; i += blockDim.x) nxt[i] = 0.0;
        }
        PROBE(3);
        grid_barrier(p.bar, epoch, P);
        PROBE(4);
        // ---------------- (iii) DLARFG (reading R1) --------------------------------
        if (tid == 0) {
            double nrm2 = ldcg(acc + 2 * FT_NBMAX + 0);
            double sx = ldcg(acc + 2 * FT_NBMAX + 1);
            double alpha = ldcg(acc + 2 * FT_NBMAX + 2);
            double xnorm = sqrt(nrm2);
            double tau, beta, scale;
            if (xnorm == 0.0 || c + 2 >= ihi) {
                tau = 0.0;
                beta = alpha;
                scale = 1.0;  // H = I, x left untouched (it is zero)
            } else {
                beta = -copysign(hypot(alpha, xnorm), alpha);
                tau = (beta - alpha) / beta;
                scale = 1.0 / (alpha - beta);
            }
            S.scal[0] = tau;
            S.scal[1] = beta;
            S.scal[2] = scale;
            S.scal[3] = alpha;
            S.scal[4] = 1.0 + scale * sx;  // V_chk(j) = e^T v
        }
        if (tid < j) S.vtb[tid] = ldcg(acc + FT_NBMAX + tid);
        __syncthreads();
        const double tau = S.scal[0], beta = S.scal[1], scale = S.scal[2], alpha = S.scal[3],
                     vchk = S.scal[4];
        if (tid < j) S.t[tid] = ldcg(V + (c + 1) + (int64_t)tid * ldw) + scale * S.vtb[tid];
        // store V(:, j) and the reduced column c of A for own rows
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
            if (cache) Vl[tid + j * ls] = vv;
            A[row + (int64_t)c * ldw] = av;
        } else if (cache && mine) {
            Vl[tid + j * ls] = 0.0;  // rows outside the panel take no part in the V^T b dots
        }
        PROBE(5);
        // ---------------- (iv) the trailing GEMV, v staged in shared memory ------------
        const bool vfy = (j == 0) && p.verify;
        const int cend = vfy ? n : ihi;
        double2 ya = make_double2(0.0, 0.0), rs = make_double2(0.0, 0.0);
        for (int cs = c + 1; cs < cend; cs += VCH) {
            const int ce = min(cend, cs + VCH);
            __syncthreads();
            for (int q = cs + tid; q < ce; q += blockDim.x)
                S.vch[q - cs] = q == c + 1 ? 1.0 : (q < ihi ? scale * ldcg(p.bvec + q) : 0.0);
            __syncthreads();
            if (gemv_on) {
                int col = cs + cl;
                for (; col + 7 * ncl < ce; col += 8 * ncl) {
                    double2 a[8];
#pragma unroll
                    for (int u = 0; u < 8; u++) a[u] = A2[(int64_t)(col + u * ncl) * ldw2 + rp];
#pragma unroll
                    for (int u = 0; u < 8; u++) {
                        const double v = S.vch[col + u * ncl - cs];
                        ya.x += a[u].x * v;
                        ya.y += a[u].y * v;
                        if (vfy) {
                            rs.x += a[u].x;
                            rs.y += a[u].y;
                        }
                    }
                }
                for (; col < ce; col += ncl) {
                    double2 a = A2[(int64_t)col * ldw2 + rp];
                    const double v = S.vch[col - cs];
                    ya.x += a.x * v;
                    ya.y += a.y * v;
                    if (vfy) {
                        rs.x += a.x;
                        rs.y += a.y;
                    }
                }
            }
        }
        PROBE(6);
        if (gemv_on) {
            S.redy[tid] = ya;
            if (vfy) S.reds[tid] = rs;
        }
        __syncthreads();
        for (int q = wid; q < R2; q += nw) {
            double sx = 0.0, sy = 0.0, tx = 0.0, ty = 0.0;
            for (int l = lane; l < ncl; l += 32) {
                double2 u = S.redy[l * R2 + q];
                sx += u.x;
                sy += u.y;
                if (vfy) {
                    double2 z = S.reds[l * R2 + q];
                    tx += z.x;
                    ty += z.y;
                }
            }
            sx = warp_sum(sx);
            sy = warp_sum(sy);
            if (vfy) {
                tx = warp_sum(tx);
                ty = warp_sum(ty);
            }
            if (lane == 0) {
                S.y2[q] = make_double2(sx, sy);
                if (vfy) S.rs2[q] = make_double2(tx, ty);
            }
        }
        __syncthreads();
        PROBE(7);
        // ---------------- (v) Y(:, j), T(:, j) -------------------------------------
        if (valid) {
            double2 yy2 = S.y2[tid >> 1];
            double yy = (tid & 1) ? yy2.y : yy2.x;
            for (int jp = 0; jp < j; jp++) yy -= Yl[tid + jp * ls] * S.t[jp];
            yy *= tau;
            Y[row + (int64_t)j * ldw] = yy;
            if (cache) Yl[tid + j * ls] = yy;
        }
        if (vfy && datarow) {
            // D_r(row) = r(row) - sum_{col >= k} L(row, col); columns < k are logical zero here
            double2 z = S.rs2[tid >> 1];
            double rsum = b0 + ((tid & 1) ? z.y : z.x);
            double d = A[row + (int64_t)n * ldw] - rsum;
            if (not_within(d, tau_abs)) {
                atomicAdd(&p.ctl->nflag, 1);
            } else if (tau_abs > 0.0) {
                double rel = fabs(d) / (tau_abs / p.ctl->c_thr);
                atomicMax(&p.ctl->drift_bits, (unsigned long long)__double_as_longlong(rel));
            }
        }
        if (tid < j) {
            double sacc = 0.0;
            for (int bb = tid; bb < j; bb++) sacc += S.Ts[tid + bb * FT_NBMAX] * S.t[bb];
            S.vtb[tid] = -tau * sacc;  // reuse vtb as scratch
        }
        __syncthreads();
        if (tid < j) S.Ts[tid + j * FT_NBMAX] = S.vtb[tid];
        if (tid == 0) {
            S.Ts[j + j * FT_NBMAX] = tau;
            if (blockIdx.x == 0) {
                p.tau[c] = tau;
                if (p.abft) {
                    p.Qc[c] = vchk - 1.0;      // Q column checksum
                    p.Qc[n] += vchk - 1.0;     // corner of the Q checksums
                }
            }
        }
        __syncthreads();
        PROBE(8);
    }
    // Q row checksums of the new Householder vectors (Fig. 5): own data rows
    if (p.abft && datarow) {
        double sacc = 0.0;
        for (int jj = 0; jj < ib; jj++)
            if (row >= k + jj + 2) sacc += Vl[tid + jj * ls];
        p.Qr[row] += sacc;
    }
    if (blockIdx.x == 0)
        for (int i = tid; i < ib * ib; i += blockDim.x) {
            int a = i % ib, bb = i / ib;
            p.T[a + bb * FT_NBMAX] = S.Ts[a + bb * FT_NBMAX];
        }
}

cudaError_t ft_launch_panel(const PanelParams &p, int nsm, cudaStream_t s) {
    static int max_smem = 0;
    if (!max_smem) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        cudaError_t e = cudaFuncSetAttribute(k_panel, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem);
        if (e != cudaSuccess) return e;
    }
    int grid = nsm < p.ngroups ? nsm : p.ngroups;
    if (grid < 1) grid = 1;
    // rows per CTA (max over CTAs) and whether their V/Y rows fit next to the fixed part
    int gmax = (p.ngroups + grid - 1) / grid;
    int rmax = 16 * gmax;
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
    return cudaLaunchCooperativeKernel((void *)k_panel, dim3(grid), dim3(PT), args, smem, s);
}
