// ft_panel.cu -- persistent DLAHR2 panel kernel (the method's hot spot).
//
// One cooperative launch factorizes one panel of ib columns (DLAHR2, Alg. 2 l.4 /
// Alg. 3 l.5; LAPACK reading R2).  For column c = k + j:
//   (i)   b0 = A(k+1:n, c) - Y(k+1:n, 0:j) V(c, 0:j)^T                [row-local]
//   (ii)  b  = b0 - V T^T (V^T b0)                                    [grid sync #1: s1 = V^T b0]
//   (iii) DLARFG on (b(c+1), b(c+2:n)) -> beta, tau, v                [grid sync #2: ||x||^2, V^T x, e^T x]
//   (iv)  y = A(k+1:n, c+1:ihi) v   -- the trailing GEMV, ~83% of the  [row-split, no reduction]
//         roofline time of the whole reduction
//   (v)   t = V^T v, Y(:, j) = tau (y - Y t), T(0:j, j) = -tau T t, T(j,j) = tau
// With ABFT the checksum row n rides as one more row of b / Y / V (V_aug(n,:) =
// e^T V = V_chk, Y_aug(n,:) = e^T Y = Y_chk; Alg. 3 l.6-7, readings R7/R8), and the
// first GEMV of the panel also produces row sums of the trailing matrix, so the
// row-checksum discrepancy D_r = r - L e is evaluated BEFORE the panel's output is
// consumed by the updates (verify-before-consume, reading R11/R14).
//
// Latency design (the column chain is serial: n-2 dependent steps, SURVEY 7 "hard parts"):
//  * rows [rbase, rend) are split into 8-row groups, contiguous per CTA; each CTA owns
//    its rows for the whole panel (b, V, Y rows cached in shared memory), so y needs no
//    cross-CTA reduction and every small dot is a CTA partial + one fp64 atomic;
//  * exactly two grid syncs per column, each followed by ONE L2 round trip;
//  * the GEMV starts right after sync #2 on the UNSCALED b,
//        y = A(:, c+1) + scale * A(:, c+2:ihi) b(c+2:ihi),   scale = 1/(alpha - beta),
//    while warp 0 evaluates DLARFG, so the reflector scalars are off the critical path;
//  * accumulator sets are indexed by the global column (mod 4) and recycled in-kernel,
//    barrier counters alternate between consecutive panel launches: no memsets per panel.
#include "ft_common.cuh"
#include "ft_internal.h"

#define PT 512        // threads per CTA
#define NW (PT / 32)  // warps per CTA
#define GR 8          // row-group granularity (64 bytes of a column)
#define VS 65         // shared-memory row stride of the V / Y row caches (doubles)
#define RMAX PT       // max rows per CTA

// accumulator set layout (FT_ACC_STRIDE doubles): [0,64) s1 = V^T b0 | [64,128) V^T x |
// 128 ||x||^2 | 129 e^T x | 130 alpha
#define ACC_VTB 64
#define ACC_NRM 128
#define ACC_SX 129
#define ACC_ALPHA 130

struct PanelSmem {
    double Ts[FT_NBMAX][FT_NBMAX + 1];  // Ts[a][b] = T(a, b)
    double vrow[FT_NBMAX];              // V(c, 0:j) of the current column
    double w[FT_NBMAX];                 // T^T s1
    double t[FT_NBMAX];                 // V^T v
    double scal[8];                     // tau, beta, scale, vchk, alpha
    double bsm[RMAX];                   // b of the own rows (masked) for the column dots
    double2 red[PT];                    // GEMV partials  (y pairs)
    double2 rsr[PT];                    // GEMV partials  (row sums, verify pass)
    // followed (dynamic part) by the CTA's rows of V and Y when they fit: [R][VS] each
};

size_t ft_panel_smem_bytes() { return sizeof(PanelSmem); }

#define PROBE(slot)                                                                   \
    do {                                                                              \
        if (p.dbg && blockIdx.x == 0 && tid == 0 && j < 64)                           \
            p.dbg[j * 16 + (slot)] = clock64();                                       \
    } while (0)

// sum over the L lanes of an aligned lane group (L a power of two <= 32)
__device__ __forceinline__ double group_sum(double v, int L) {
#pragma unroll 1
    for (int o = L >> 1; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// DLARFG scalars (reading R1), out of line: one copy of the sqrt / division code
struct Refl {
    double tau, beta, scale;
};
__device__ __noinline__ Refl dlarfg_scalars(double nrm2, double alpha, bool trivial) {
    Refl r;
    if (nrm2 == 0.0 || trivial) {
        r.tau = 0.0;  // H = I, x left untouched (it is zero)
        r.beta = alpha;
        r.scale = 1.0;
    } else {
        r.beta = -copysign(sqrt(alpha * alpha + nrm2), alpha);  // -sign(alpha) hypot(alpha, ||x||)
        r.tau = (r.beta - alpha) / r.beta;
        r.scale = 1.0 / (alpha - r.beta);
    }
    return r;
}

// lanes per output for J column dots (L * J <= PT), as log2
__device__ __forceinline__ int coldot_log2L(int J) { return J <= 16 ? 5 : (J <= 32 ? 4 : (J <= 64 ? 3 : 2)); }

__device__ __forceinline__ int pow2_floor(int x) {
    int p = 1;
    while (p * 2 <= x) p *= 2;
    return p;
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
    const int r0 = p.rbase + GR * g0, r1 = p.rbase + GR * g1;
    const int R = r1 - r0, R2 = R >> 1;
    const int n = p.n, ihi = p.ihi, k = p.k, ib = p.ib;
    const int64_t ldw = p.ldw;
    double *__restrict__ A = p.A;
    double *__restrict__ V = p.V;
    double *__restrict__ Y = p.Y;
    unsigned epoch = 0;
    if (blockIdx.x == 0 && tid == 0) *p.bar_next = 0u;  // the next panel launch's counter

    // own rows of V and Y: [rl][jp] in shared memory (write-through to global) when they fit
    double *Vl = CACHE ? reinterpret_cast<double *>(smem_raw + sizeof(PanelSmem)) : V + r0;
    double *Yl = CACHE ? Vl + (int64_t)VS * R : Y + r0;
    constexpr int64_t XR = CACHE ? VS : 1;  // row stride
    const int64_t XC = CACHE ? 1 : ldw;     // column stride

    // row-dot mapping: tpr lanes per own row
    const int tpr = min(8, pow2_floor(PT / R));
    const int tsh = __ffs(tpr) - 1;
    const int rl = tid >> tsh, lr = tid & (tpr - 1);
    const int row = r0 + rl;
    const bool mine = rl < R;
    const bool datarow = mine && row >= k + 1 && row < ihi;
    const bool chkrow = mine && p.abft && row == n;
    const bool valid = datarow || chkrow;
    const bool leader = mine && lr == 0;

    // GEMV mapping: row pair rp, column lane cl (R2p lanes per column; pow2 when <= 32 so
    // the lanes of one row pair are shuffle-reducible inside a warp)
    int R2p = R2;
    if (R2 <= 32) {
        R2p = 1;
        while (R2p < R2) R2p *= 2;
    }
    const int ncl = PT / R2p;
    const int rp = tid % R2p, cl = tid / R2p;
    const bool gemv_on = rp < R2 && cl < ncl;
    const int npart = R2p <= 32 ? NW : ncl;  // partials per row pair after the warp stage
    const double2 *__restrict__ A2 = reinterpret_cast<const double2 *>(A + r0);
    const int64_t ldw2 = ldw >> 1;

    const double c_thr = p.ctl->c_thr;
    const double tau_abs = c_thr * (double)n * 2.220446049250313e-16 * p.ctl->normF;

#pragma unroll 1
    for (int i = tid; i < FT_NBMAX * (FT_NBMAX + 1); i += PT) (&S.Ts[0][0])[i] = 0.0;
    double acol = (leader && valid) ? A[row + (int64_t)k * ldw] : 0.0;  // A(row, c)
    __syncthreads();

    for (int j = 0; j < ib; j++) {
        const int c = k + j;
        double *acc = p.acc + (c & 3) * FT_ACC_STRIDE;
        // A(row, c+1): the first term of y, and the next column's acol (column c+1 is not
        // modified while column c is processed)
        const double anext = (leader && valid) ? A[row + (int64_t)(c + 1) * ldw] : 0.0;
        PROBE(0);
        // ---------------- (i) b0 = A(:,c) - Y V(c,:)^T ------------------------------------
        double b0 = acol;
        if (j > 0) {
            double sacc = 0.0;
            if (mine)
#pragma unroll 1
                for (int jp = lr; jp < j; jp += tpr) sacc += Yl[rl * XR + jp * XC] * S.vrow[jp];
            b0 = acol - group_sum(sacc, tpr);
            if (leader) S.bsm[rl] = datarow ? b0 : 0.0;
            __syncthreads();
            // s1 = V^T b0 over the data rows: one partial per CTA and output
            {
                const int lg = coldot_log2L(j), L = 1 << lg;
                const int o = tid >> lg, lc = tid & (L - 1);
                double s = 0.0;
                if (o < j)
#pragma unroll 1
                    for (int t2 = lc; t2 < R; t2 += L) s += Vl[t2 * XR + o * XC] * S.bsm[t2];
                s = group_sum(s, L);
                if (o < j && lc == 0 && !(p.dbg_mode & 4)) atomicAdd(acc + o, s);
            }
            PROBE(1);
            if (!(p.dbg_mode & 1)) grid_barrier(p.bar, epoch, P);
            PROBE(2);
            // w = T^T s1 (8 lanes per output, s1 read straight from L2)
            {
                const int a = tid >> 3, q = tid & 7;
                double s = 0.0;
#pragma unroll
                for (int u = 0; u < FT_NBMAX / 8; u++) {
                    const int bb = q + 8 * u;
                    if (a < j && bb <= a) s += S.Ts[bb][a] * ldcg(acc + bb);
                }
                s += __shfl_xor_sync(0xffffffffu, s, 1);
                s += __shfl_xor_sync(0xffffffffu, s, 2);
                s += __shfl_xor_sync(0xffffffffu, s, 4);
                if (a < j && q == 0) S.w[a] = s;
            }
            __syncthreads();
            PROBE(3);
        }
        // ---------------- (ii) b = b0 - V w --------------------------------------------------
        double b = b0;
        if (j > 0) {
            double sacc = 0.0;
            if (mine)
#pragma unroll 1
                for (int jp = lr; jp < j; jp += tpr) sacc += Vl[rl * XR + jp * XC] * S.w[jp];
            b = b0 - group_sum(sacc, tpr);
        }
        const bool xrow = datarow && row >= c + 2;
        if (leader) {
            S.bsm[rl] = xrow ? b : 0.0;
            if (xrow) p.bvec[row] = b;
            if (datarow && row == c + 1) acc[ACC_ALPHA] = b;  // alpha: a single writer
        }
        __syncthreads();
        // V^T x (jp < j), ||x||^2 (jp = j), e^T x (jp = j + 1) over the own x rows
        {
            const int J = j + 2;
            const int lg = coldot_log2L(J), L = 1 << lg;
            const int o = tid >> lg, lc = tid & (L - 1);
            double s = 0.0;
            if (o < J)
#pragma unroll 1
                for (int t2 = lc; t2 < R; t2 += L) {
                    const double bt = S.bsm[t2];
                    s += (o < j ? Vl[t2 * XR + o * XC] : (o == j ? bt : 1.0)) * bt;
                }
            s = group_sum(s, L);
            if (o < J && lc == 0 && !(p.dbg_mode & 4))
                atomicAdd(acc + (o < j ? ACC_VTB + o : (o == j ? ACC_NRM : ACC_SX)), s);
        }
        PROBE(4);
        if (!(p.dbg_mode & 1)) grid_barrier(p.bar, epoch, P);
        PROBE(5);
        // ---------------- (iii) DLARFG (reading R1) in warp 0, concurrent with the GEMV -------
        if (wid == 0) {
            const double nrm2 = ldcg(acc + ACC_NRM), sx = ldcg(acc + ACC_SX), alpha = ldcg(acc + ACC_ALPHA);
            double vn0 = 0.0, vt0 = 0.0, vn1 = 0.0, vt1 = 0.0;
            if (lane < j) {
                vn0 = ldcg(V + (c + 1) + (int64_t)lane * ldw);
                vt0 = ldcg(acc + ACC_VTB + lane);
            }
            if (lane + 32 < j) {
                vn1 = ldcg(V + (c + 1) + (int64_t)(lane + 32) * ldw);
                vt1 = ldcg(acc + ACC_VTB + lane + 32);
            }
            const Refl rf = dlarfg_scalars(nrm2, alpha, c + 2 >= ihi);
            const double tau = rf.tau, beta = rf.beta, scale = rf.scale;
            // t = V^T v = V(c+1,:)^T + scale * V^T x; V(c+1, :) is also the next column's vrow
            if (lane < j) {
                S.t[lane] = vn0 + scale * vt0;
                S.vrow[lane] = vn0;
            }
            if (lane + 32 < j) {
                S.t[lane + 32] = vn1 + scale * vt1;
                S.vrow[lane + 32] = vn1;
            }
            if (lane == 0) {
                S.vrow[j] = 1.0;
                S.scal[0] = tau;
                S.scal[1] = beta;
                S.scal[2] = scale;
                S.scal[3] = 1.0 + scale * sx;  // V_chk(j) = e^T v
                S.scal[4] = alpha;
            }
        }
        PROBE(6);
        // ---------------- (iv) the trailing GEMV on the unscaled b ---------------------------
        const bool vfy = (j == 0) && p.verify;
        const int cend = vfy ? n : ihi;
        double2 ya = make_double2(0.0, 0.0), rs = make_double2(0.0, 0.0);
        if (gemv_on && !(p.dbg_mode & 2)) {
            const double *bv = p.bvec;  // b(q) for c+2 <= q < ihi; zero for q >= ihi
            int col = c + 2 + cl;
#pragma unroll 1
            for (; col + 7 * ncl < cend; col += 8 * ncl) {
                double2 a[8];
                double v[8];
#pragma unroll
                for (int u = 0; u < 8; u++) {
                    const int q = col + u * ncl;
                    a[u] = A2[(int64_t)q * ldw2 + rp];
                    v[u] = ldcg(bv + q);
                }
#pragma unroll
                for (int u = 0; u < 8; u++) {
                    ya.x += a[u].x * v[u];
                    ya.y += a[u].y * v[u];
                    rs.x += a[u].x;  // row sums: used by the verify pass only (cheap, HBM-bound loop)
                    rs.y += a[u].y;
                }
            }
#pragma unroll 1
            for (; col < cend; col += ncl) {
                const double2 a = A2[(int64_t)col * ldw2 + rp];
                const double v = ldcg(bv + col);
                ya.x += a.x * v;
                ya.y += a.y * v;
                rs.x += a.x;
                rs.y += a.y;
            }
        }
        PROBE(7);
        // partials: shuffle over the lanes of a row pair inside the warp, then shared memory
        if (R2p <= 32) {
#pragma unroll
            for (int o = 1; o < 32; o <<= 1)
                if (o >= R2p) {
                    ya.x += __shfl_xor_sync(0xffffffffu, ya.x, o);
                    ya.y += __shfl_xor_sync(0xffffffffu, ya.y, o);
                    if (vfy) {
                        rs.x += __shfl_xor_sync(0xffffffffu, rs.x, o);
                        rs.y += __shfl_xor_sync(0xffffffffu, rs.y, o);
                    }
                }
            if (lane < R2p) {
                S.red[wid * R2p + lane] = ya;
                if (vfy) S.rsr[wid * R2p + lane] = rs;
            }
        } else if (cl < ncl) {
            S.red[cl * R2p + rp] = ya;
            if (vfy) S.rsr[cl * R2p + rp] = rs;
        }
        // (zero the accumulator set of column c+2 (= that of column c-2): every CTA has
        // finished reading it, and column c+2 starts adding into it after two more syncs)
        if (blockIdx.x == 0)
            for (int i = tid; i < FT_ACC_STRIDE; i += PT) p.acc[((c + 2) & 3) * FT_ACC_STRIDE + i] = 0.0;
        __syncthreads();
        PROBE(8);
        // ---------------- (v) Y(:, j), T(:, j), V(:, j), reduced column c -------------------
        const double tau = S.scal[0], scale = S.scal[2];
        {
            double sacc = 0.0;
            if (mine)
#pragma unroll 1
                for (int jp = lr; jp < j; jp += tpr) sacc += Yl[rl * XR + jp * XC] * S.t[jp];
            sacc = group_sum(sacc, tpr);
            if (leader) {
                if (valid) {
                    double yb = 0.0;
                    const int pr = rl >> 1;
#pragma unroll 1
                    for (int q = 0; q < npart; q++) {
                        const double2 u = S.red[q * R2p + pr];
                        yb += (rl & 1) ? u.y : u.x;
                    }
                    const double yy = tau * (anext + scale * yb - sacc);
                    Y[row + (int64_t)j * ldw] = yy;
                    if (CACHE) Yl[rl * XR + j * XC] = yy;
                    const double beta = S.scal[1], vchk = S.scal[3], alpha = S.scal[4];
                    double vv, av;
                    if (chkrow) {
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
                    if (CACHE) Vl[rl * XR + j * XC] = vv;
                    A[row + (int64_t)c * ldw] = av;
                    if (vfy && datarow) {
                        // D_r(row) = r(row) - sum_{col >= k} L(row, col); columns < k are logical zero
                        double rsum = 0.0;
#pragma unroll 1
                        for (int q = 0; q < npart; q++) {
                            const double2 u = S.rsr[q * R2p + pr];
                            rsum += (rl & 1) ? u.y : u.x;
                        }
                        rsum += b0 + anext;
                        const double d = A[row + (int64_t)n * ldw] - rsum;
                        if (not_within(d, tau_abs)) {
                            atomicAdd(&p.ctl->nflag, 1);
                        } else if (tau_abs > 0.0) {
                            const double rel = fabs(d) / (tau_abs / c_thr);
                            atomicMax(&p.ctl->drift_bits, (unsigned long long)__double_as_longlong(rel));
                        }
                    }
                } else if (CACHE) {
                    Vl[rl * XR + j * XC] = 0.0;  // rows outside the panel take no part in the dots
                }
            }
        }
        {   // T(a, j) = -tau * sum_{b=a}^{j-1} T(a, b) t(b), 8 lanes per output
            const int a = tid >> 3, q = tid & 7;
            double s = 0.0;
            if (a < j)
                for (int bb = a + q; bb < j; bb += 8) s += S.Ts[a][bb] * S.t[bb];
            s += __shfl_xor_sync(0xffffffffu, s, 1);
            s += __shfl_xor_sync(0xffffffffu, s, 2);
            s += __shfl_xor_sync(0xffffffffu, s, 4);
            if (a < j && q == 0) S.Ts[a][j] = -tau * s;
            if (tid == 0) S.Ts[j][j] = tau;
        }
        if (blockIdx.x == 0 && tid == 0) {
            p.tau[c] = tau;
            if (p.abft) {
                const double vchk = S.scal[3];
                p.Qc[c] = vchk - 1.0;   // Q column checksum
                p.Qc[n] += vchk - 1.0;  // corner of the Q checksums
            }
        }
        acol = anext;
        __syncthreads();
        PROBE(9);
    }
    // Q row checksums of the new Householder vectors (Fig. 5): own data rows
    if (p.abft && leader && datarow) {
        double s = 0.0;
#pragma unroll 1
        for (int jj = 0; jj < ib; jj++)
            if (row >= k + jj + 2) s += Vl[rl * XR + jj * XC];
        p.Qr[row] += s;
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
    const int gmax = (p.ngroups + grid - 1) / grid;
    const int rmax = GR * gmax;
    if (rmax > RMAX) return cudaErrorInvalidConfiguration;  // n beyond ~75k rows per GPU
    const size_t fixed = sizeof(PanelSmem);
    const size_t want = fixed + (size_t)2 * VS * rmax * sizeof(double);
    const bool cache = want <= (size_t)max_smem;
    void *args[] = {const_cast<PanelParams *>(&p)};
    g_ft_launches++;
    const void *fn = cache ? (const void *)k_panel<true> : (const void *)k_panel<false>;
    return cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(PT), args, cache ? want : fixed, s);
}

int ft_panel_group_rows() { return GR; }
