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
//  * warp 0 is the CONTROL warp: it runs the whole column chain (i)-(iii), (v) warp-
//    synchronously (lane = row for row dots, lane = output for column dots, no CTA-wide
//    barriers) and the two grid syncs per column; warps 1..15 only stream A for the
//    GEMV.  The two roles meet at two named barriers per column (GO, DONE);
//  * the GEMV runs on the UNSCALED b right after sync #2,
//        y = A(:, c+1) + scale * A(:, c+2:ihi) b(c+2:ihi),   scale = 1/(alpha - beta),
//    while the control warp evaluates DLARFG, T(:, j) and the stores of V(:, j) and the
//    reduced column, so only the Y(:, j) step follows the GEMV on the critical path;
//  * accumulator sets are indexed by the global column (mod 4) and recycled in-kernel,
//    barrier counters alternate between consecutive panel launches: no memsets per panel.
#include "ft_common.cuh"
#include "ft_internal.h"

#include <cstdlib>

#define PT 512        // threads per CTA
#define NW (PT / 32)  // warps per CTA
#define NGW (NW - 1)  // GEMV warps (warp 0 is the control warp)
#define GR 8          // row-group granularity (64 bytes of a column)
#define VS 65         // shared-memory row stride of the V / Y row caches (doubles)
#define RMAX PT       // max rows per CTA
#define BAR_GO 1      // named barrier: b(c+2:ihi) is published, start the GEMV
#define BAR_DONE 2    // named barrier: GEMV partials are in shared memory
#ifndef GB
#define GB 8          // GEMV load batch (double2 of A + b per lane)
#endif

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
    double s1[FT_NBMAX];                // V^T b0 (reduced)
    double scal[8];                     // tau, beta, scale, vchk, alpha
    double acol[RMAX];                  // A(row, c) of the own rows
    double anext[RMAX];                 // A(row, c+1)
    double b0[RMAX];                    // b0 (rows), then b
    double bm[RMAX];                    // masked b0 / x for the column dots
    double2 red[PT];                    // GEMV partials  (y pairs)
    double2 rsr[PT];                    // GEMV partials  (row sums, verify pass)
    // followed (dynamic part) by the CTA's rows of V and Y when they fit: [R][VS] each
};

size_t ft_panel_smem_bytes() { return sizeof(PanelSmem); }

#define PROBE(slot)                                                                   \
    do {                                                                              \
        if (p.dbg && blockIdx.x == 0 && lane == 0 && j < 64)                          \
            p.dbg[j * 16 + (slot)] = clock64();                                       \
    } while (0)

__device__ __forceinline__ void named_bar(int id) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(PT) : "memory"); }

// grid barrier driven by one warp: lane 0 arrives (release) and polls (acquire); the
// warp-level barriers order the other lanes' accesses around it
__device__ __forceinline__ void warp_grid_barrier(unsigned *count, unsigned &epoch, unsigned nblocks) {
    __syncwarp();
    if ((threadIdx.x & 31) == 0) {
        epoch += 1;
        const unsigned target = epoch * nblocks;
        red_release_add_u32(count, 1u);
        while (ld_acquire_u32(count) < target) {
        }
    }
    __syncwarp();
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

// sum_{jp < J} X[jp * cs] * z[jp] with four independent chains
__device__ __forceinline__ double dotj(const double *X, int64_t cs, const double *z, int J) {
    double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
    int jp = 0;
#pragma unroll 1
    for (; jp + 3 < J; jp += 4) {
        s0 += X[jp * cs] * z[jp];
        s1 += X[(jp + 1) * cs] * z[jp + 1];
        s2 += X[(jp + 2) * cs] * z[jp + 2];
        s3 += X[(jp + 3) * cs] * z[jp + 3];
    }
#pragma unroll 1
    for (; jp < J; jp++) s0 += X[jp * cs] * z[jp];
    return (s0 + s1) + (s2 + s3);
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

    // own rows of V and Y: [rl][jp] in shared memory (write-through to global) when they fit
    double *Vl = CACHE ? reinterpret_cast<double *>(smem_raw + sizeof(PanelSmem)) : V + r0;
    double *Yl = CACHE ? Vl + (int64_t)VS * R : Y + r0;
    constexpr int64_t XR = CACHE ? VS : 1;  // row stride
    const int64_t XC = CACHE ? 1 : ldw;     // column stride

    // GEMV partial layout (shared by both roles): R2p lanes per column, a power of two
    // when <= 32 so the lanes of one row pair are shuffle-reducible inside a warp
    int R2p = R2;
    if (R2 <= 32) {
        R2p = 1;
        while (R2p < R2) R2p *= 2;
    }
    const int ncl = (NGW * 32) / R2p;
    const int npart = R2p <= 32 ? NGW : ncl;  // partials per row pair

#pragma unroll 1
    for (int i = tid; i < FT_NBMAX * (FT_NBMAX + 1); i += PT) (&S.Ts[0][0])[i] = 0.0;
    if (p.ckpt) {
        // diskless checkpoint of the panel columns, r, c, kappa, Qr, Qc, Fr, taken
        // before anything is modified: own rows by their owner, c by the owner of row n (it
        // rewrites c(k:e)), the rest grid-strided; all of it precedes this CTA's first arrival
        const int rend = p.abft ? n + 1 : ihi;
        for (int x = tid; x < R * ib; x += PT) {
            const int rl = x % R, jj = x / R, row = r0 + rl;
            if (row < rend) p.ckpt[row + (int64_t)jj * ldw] = A[row + (int64_t)(k + jj) * ldw];
        }
        const int gstride = (int)P * PT, g = blockIdx.x * PT + tid;
        for (int x = g; x < p.rbase * ib; x += gstride) {
            const int i = x % p.rbase, jj = x / p.rbase;
            p.ckpt[i + (int64_t)jj * ldw] = A[i + (int64_t)(k + jj) * ldw];
        }
        for (int i = g; i <= n; i += gstride) {
            p.ck_r[i] = A[i + (int64_t)n * ldw];
            p.ck_q[i] = p.Qr[i];
            p.ck_q[ldw + i] = p.Qc[i];
            p.ck_q[2 * ldw + i] = p.Fr[i];
        }
        if (r0 <= n && n < r1)
            for (int i = tid; i <= n; i += PT) p.ck_c[i] = A[n + (int64_t)i * ldw];
    }
    for (int rl = tid; rl < R; rl += PT) {
        const int row = r0 + rl;
        const bool valid = (row >= k + 1 && row < ihi) || (p.abft && row == n);
        S.acol[rl] = valid ? A[row + (int64_t)k * ldw] : 0.0;
    }
    __syncthreads();

    if (wid > 0) {
        // ======================= GEMV warps =============================================
        const int gt = tid - 32;
        const int rp = gt % R2p, cl = gt / R2p;
        const bool gemv_on = rp < R2 && cl < ncl;
        const double2 *__restrict__ A2 = reinterpret_cast<const double2 *>(A + r0);
        const int64_t ldw2 = ldw >> 1;
        const double *bv = p.bvec;  // b(q) for c+2 <= q < ihi; zero for q >= ihi
#pragma unroll 1
        for (int j = 0; j < ib; j++) {
            const int c = k + j;
            const bool vfy = (j == 0) && p.verify;
            const int cend = vfy ? n : ihi;
            named_bar(BAR_GO);
            double2 ya = make_double2(0.0, 0.0), rs = make_double2(0.0, 0.0);
            if (gemv_on && !(p.dbg_mode & 2)) {
                // b is read with plain (L1-allocating) loads: the control warp's acquire at
                // sync #2 invalidated this SM's L1 (CCTL.IVALL) before BAR_GO released us
                int col = c + 2 + cl;
#pragma unroll 1
                for (; col + (GB - 1) * ncl < cend; col += GB * ncl) {
                    double2 a[GB];
                    double v[GB];
#pragma unroll
                    for (int u = 0; u < GB; u++) {
                        const int q = col + u * ncl;
                        a[u] = A2[(int64_t)q * ldw2 + rp];
                        v[u] = bv[q];
                    }
#pragma unroll
                    for (int u = 0; u < GB; u++) {
                        ya.x += a[u].x * v[u];
                        ya.y += a[u].y * v[u];
                        rs.x += a[u].x;  // row sums: used by the verify pass only (cheap, memory-bound loop)
                        rs.y += a[u].y;
                    }
                }
#pragma unroll 1
                for (; col < cend; col += ncl) {
                    const double2 a = A2[(int64_t)col * ldw2 + rp];
                    const double v = bv[col];
                    ya.x += a.x * v;
                    ya.y += a.y * v;
                    rs.x += a.x;
                    rs.y += a.y;
                }
            }
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
                    S.red[(wid - 1) * R2p + lane] = ya;
                    if (vfy) S.rsr[(wid - 1) * R2p + lane] = rs;
                }
            } else if (cl < ncl) {
                S.red[cl * R2p + rp] = ya;
                if (vfy) S.rsr[cl * R2p + rp] = rs;
            }
            named_bar(BAR_DONE);
        }
        return;
    }

    // ======================= control warp =================================================
    unsigned epoch = 0;
    if (blockIdx.x == 0 && lane == 0) *p.bar_next = 0u;  // the next panel launch's counter
    const double c_thr = p.ctl->c_thr;
    const double tau_abs = c_thr * (double)n * 2.220446049250313e-16 * p.ctl->normF;
    auto is_data = [&](int row) { return row >= k + 1 && row < ihi; };
    auto is_valid = [&](int row) { return (row >= k + 1 && row < ihi) || (p.abft && row == n); };

#pragma unroll 1
    for (int j = 0; j < ib; j++) {
        const int c = k + j;
        double *acc = p.acc + (c & 3) * FT_ACC_SET_DOUBLES;  // accumulator i at acc[i * FT_ACC_PAD]
        // A(row, c+1) of the first two row chunks: issued now, consumed after the GEMV
        double an0 = 0.0, an1 = 0.0;
        if (lane < R && is_valid(r0 + lane)) an0 = A[(r0 + lane) + (int64_t)(c + 1) * ldw];
        if (lane + 32 < R && is_valid(r0 + lane + 32)) an1 = A[(r0 + lane + 32) + (int64_t)(c + 1) * ldw];
        PROBE(0);
        // ---------------- (i) b0 = A(:,c) - Y V(c,:)^T, s1 = V^T b0 -----------------------
        if (j > 0) {
#pragma unroll 1
            for (int rl = lane; rl < R; rl += 32) {
                const double b0 = S.acol[rl] - dotj(Yl + rl * XR, XC, S.vrow, j);
                S.b0[rl] = b0;
                S.bm[rl] = is_data(r0 + rl) ? b0 : 0.0;
            }
            __syncwarp();
#pragma unroll 1
            for (int o = lane; o < j; o += 32) {
                const double s = dotj(Vl + o * XC, XR, S.bm, R);
                if (!(p.dbg_mode & 4)) atomicAdd(acc + o * FT_ACC_PAD, s);
            }
            PROBE(1);
            if (!(p.dbg_mode & 1)) warp_grid_barrier(p.bar, epoch, P);
            PROBE(2);
            // w = T^T s1
            if (lane < j) S.s1[lane] = ldcg(acc + lane * FT_ACC_PAD);
            if (lane + 32 < j) S.s1[lane + 32] = ldcg(acc + (lane + 32) * FT_ACC_PAD);
            __syncwarp();
#pragma unroll 1
            for (int a = lane; a < j; a += 32) S.w[a] = dotj(&S.Ts[0][a], FT_NBMAX + 1, S.s1, a + 1);
            __syncwarp();
            // ---------------- (ii) b = b0 - V w ---------------------------------------------
#pragma unroll 1
            for (int rl = lane; rl < R; rl += 32) S.b0[rl] -= dotj(Vl + rl * XR, XC, S.w, j);
        } else {
#pragma unroll 1
            for (int rl = lane; rl < R; rl += 32) S.b0[rl] = S.acol[rl];
        }
        PROBE(3);
        // publish x = b(c+2:ihi) for the GEMV, alpha = b(c+1); column dots of x
#pragma unroll 1
        for (int rl = lane; rl < R; rl += 32) {
            const int row = r0 + rl;
            const double b = S.b0[rl];
            const bool xrow = is_data(row) && row >= c + 2;
            S.bm[rl] = xrow ? b : 0.0;
            if (xrow) p.bvec[row] = b;
            if (row == c + 1) acc[ACC_ALPHA * FT_ACC_PAD] = b;  // alpha: a single writer
        }
        __syncwarp();
#pragma unroll 1
        for (int o = lane; o < j + 2; o += 32) {
            double s;
            if (o < j) s = dotj(Vl + o * XC, XR, S.bm, R);
            else if (o == j) s = dotj(S.bm, 1, S.bm, R);
            else {
                s = 0.0;
                for (int rl = 0; rl < R; rl++) s += S.bm[rl];
            }
            if (!(p.dbg_mode & 4)) atomicAdd(acc + (o < j ? ACC_VTB + o : (o == j ? ACC_NRM : ACC_SX)) * FT_ACC_PAD, s);
        }
        PROBE(4);
        if (!(p.dbg_mode & 1)) warp_grid_barrier(p.bar, epoch, P);
        PROBE(5);
        named_bar(BAR_GO);  // the GEMV warps start on the unscaled b
        // ---------------- (iii) DLARFG (reading R1), concurrent with the GEMV ---------------
        {
            const double nrm2 = ldcg(acc + ACC_NRM * FT_ACC_PAD), sx = ldcg(acc + ACC_SX * FT_ACC_PAD),
                         alpha = ldcg(acc + ACC_ALPHA * FT_ACC_PAD);
            double vn0 = 0.0, vt0 = 0.0, vn1 = 0.0, vt1 = 0.0;
            if (lane < j) {
                vn0 = ldcg(V + (c + 1) + (int64_t)lane * ldw);
                vt0 = ldcg(acc + (ACC_VTB + lane) * FT_ACC_PAD);
            }
            if (lane + 32 < j) {
                vn1 = ldcg(V + (c + 1) + (int64_t)(lane + 32) * ldw);
                vt1 = ldcg(acc + (ACC_VTB + lane + 32) * FT_ACC_PAD);
            }
            const Refl rf = dlarfg_scalars(nrm2, alpha, c + 2 >= ihi);
            const double tau = rf.tau, beta = rf.beta, scale = rf.scale;
            const double vchk = 1.0 + scale * sx;  // V_chk(j) = e^T v
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
                S.scal[2] = scale;
            }
            __syncwarp();
            // T(a, j) = -tau * sum_{b=a}^{j-1} T(a, b) t(b), T(j, j) = tau
#pragma unroll 1
            for (int a = lane; a < j; a += 32) S.Ts[a][j] = -tau * dotj(&S.Ts[a][a], 1, S.t + a, j - a);
            if (lane == 0) S.Ts[j][j] = tau;
            // V(:, j) and the reduced column c of the own rows
#pragma unroll 1
            for (int rl = lane; rl < R; rl += 32) {
                const int row = r0 + rl;
                const double b = S.b0[rl];
                if (row == n && p.abft) {
                    V[row + (int64_t)j * ldw] = vchk;
                    if (CACHE) Vl[rl * XR + j * XC] = vchk;
                    A[row + (int64_t)c * ldw] = (tau != 0.0) ? b - vchk * (alpha - beta) : b;  // left term (R7)
                } else if (is_data(row)) {
                    double vv, av;
                    if (row <= c) {
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
                } else if (CACHE) {
                    Vl[rl * XR + j * XC] = 0.0;  // rows outside the panel take no part in the dots
                }
            }
            if (blockIdx.x == 0 && lane == 0) {
                p.tau[c] = tau;
                if (p.abft) {
                    p.Qc[c] = vchk - 1.0;   // Q column checksum
                    p.Qc[n] += vchk - 1.0;  // corner of the Q checksums
                }
            }
            // recycle the accumulator set of column c+2 (= that of column c-2): every CTA has
            // finished reading it, and column c+2 adds into it only after two more syncs
            if (blockIdx.x == 0)
                for (int i = lane; i < FT_ACC_STRIDE; i += 32) p.acc[((c + 2) & 3) * FT_ACC_SET_DOUBLES + i * FT_ACC_PAD] = 0.0;
            if (lane < R) S.anext[lane] = an0;
            if (lane + 32 < R) S.anext[lane + 32] = an1;
            for (int rl = lane + 64; rl < R; rl += 32)
                S.anext[rl] = is_valid(r0 + rl) ? A[(r0 + rl) + (int64_t)(c + 1) * ldw] : 0.0;
        }
        PROBE(6);
        named_bar(BAR_DONE);  // GEMV partials ready
        PROBE(7);
        // ---------------- (v) Y(:, j) = tau (y - Y t) ----------------------------------------
        {
            const double tau = S.scal[0], scale = S.scal[2];
            const bool vfy = (j == 0) && p.verify;
#pragma unroll 1
            for (int rl = lane; rl < R; rl += 32) {
                const int row = r0 + rl;
                const double an = S.anext[rl];
                if (is_valid(row)) {
                    const int pr = rl >> 1;
                    double y0 = 0.0, y1 = 0.0;
                    int q = 0;
#pragma unroll 1
                    for (; q + 1 < npart; q += 2) {
                        const double2 u0 = S.red[q * R2p + pr], u1 = S.red[(q + 1) * R2p + pr];
                        y0 += (rl & 1) ? u0.y : u0.x;
                        y1 += (rl & 1) ? u1.y : u1.x;
                    }
                    if (q < npart) {
                        const double2 u0 = S.red[q * R2p + pr];
                        y0 += (rl & 1) ? u0.y : u0.x;
                    }
                    const double yy = tau * (an + scale * (y0 + y1) - dotj(Yl + rl * XR, XC, S.t, j));
                    Y[row + (int64_t)j * ldw] = yy;
                    if (CACHE) Yl[rl * XR + j * XC] = yy;
                    if (vfy && is_data(row)) {
                        // D_r(row) = r(row) - sum_{col >= k} L(row, col); columns < k are logical zero
                        double rsum = 0.0;
                        for (int q2 = 0; q2 < npart; q2++) {
                            const double2 u = S.rsr[q2 * R2p + pr];
                            rsum += (rl & 1) ? u.y : u.x;
                        }
                        rsum += S.acol[rl] + an;
                        const double d = A[row + (int64_t)n * ldw] - rsum;
                        if (not_within(d, tau_abs)) {
                            atomicAdd(&p.ctl->nflag, 1);
                        } else if (tau_abs > 0.0) {
                            const double rel = fabs(d) / (tau_abs / c_thr);
                            atomicMax(&p.ctl->drift_bits, (unsigned long long)__double_as_longlong(rel));
                        }
                    }
                }
                S.acol[rl] = an;
            }
            __syncwarp();
        }
        PROBE(8);
    }
    // Q row checksums of the new Householder vectors (Fig. 5): own data rows
    if (p.abft)
        for (int rl = lane; rl < R; rl += 32) {
            const int row = r0 + rl;
            if (!is_data(row)) continue;
            double s = 0.0;
            for (int jj = 0; jj < ib; jj++)
                if (row >= k + jj + 2) s += Vl[rl * XR + jj * XC];
            p.Qr[row] += s;
        }
    if (p.precheck_sums)  // e^T Y, e^T V over the own data rows (pre-update check R15, fused)
        for (int jj = lane; jj < ib; jj += 32) {
            double sy = 0.0, sv = 0.0;
            for (int rl = 0; rl < R; rl++)
                if (is_data(r0 + rl)) {
                    sy += Yl[rl * XR + jj * XC];
                    sv += Vl[rl * XR + jj * XC];
                }
            atomicAdd(&p.ctl->eY[jj], sy);
            atomicAdd(&p.ctl->eV[jj], sv);
        }
    if (blockIdx.x == 0)
        for (int i = lane; i < ib * ib; i += 32) {
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
    static int ctas = -1;
    if (ctas < 0) {
        const char *e = getenv("FT_PANEL_CTAS");  // experiment knob: cap on the panel grid
        ctas = e ? atoi(e) : 0;
    }
    if (ctas > 0 && ctas < nsm) nsm = ctas;
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
