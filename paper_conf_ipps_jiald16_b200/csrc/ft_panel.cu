// ft_panel.cu -- persistent DLAHR2 panel kernel (the method's hot spot).
//
// One cooperative launch factorizes one panel of ib columns (DLAHR2, Alg. 2 l.4 /
// Alg. 3 l.5; LAPACK reading R2).  For column c = k + j:
//   (i)   b0 = A(k+1:n, c) - Y(k+1:n, 0:j) V(c, 0:j)^T                [row-local]
//   (ii)  b  = b0 - V T^T (V^T b0)
//   (iii) DLARFG on (b(c+1), b(c+2:n)) -> beta, tau, v
//   (iv)  y = A(k+1:n, c+1:ihi) v   -- the trailing GEMV, ~83% of the roofline time of the
//         whole reduction
//   (v)   t = V^T v, Y(:, j) = tau (y - Y t), T(0:j, j) = -tau T t, T(j,j) = tau
// With ABFT the checksum row n rides as one more row of b / Y / V (V_aug(n,:) =
// e^T V = V_chk, Y_aug(n,:) = e^T Y = Y_chk; Alg. 3 l.6-7, readings R7/R8), and the
// first GEMV of the panel also produces row sums of the trailing matrix, so the
// row-checksum discrepancy D_r = r - L e is evaluated BEFORE the panel's output is
// consumed by the updates (verify-before-consume, reading R11/R14).
//
// ONE grid-wide reduction per column (the column chain is serial: n-2 dependent steps, and a
// grid sync with its reduction costs ~2 us on B200, profiles/r01/mb_sync*.txt, mb_ll.txt).
// Steps (ii)-(iii) are evaluated from b0 alone: the CTAs reduce s1 = V^T b0, sx = V_x^T b0_x,
// bb = ||b0_x||^2 and e^T b0_x (x = rows >= c+2), and every CTA derives, with w = T^T s1,
//     ||x||^2 = bb - 2 w.sx + w^T G w,   G = V_x^T V_x (Gram, carried and downdated per column)
//     alpha = b0(c+1) - V(c+1,:) w,      t = V^T v = V(c+1,:)^T + scale (sx - G w)
// and the GEMV runs on b0 itself (it was published before the sync):
//     y = A(:, c+1) + scale (A(:, c+2:) b0_x - Z w),   Z = A(:, c+2:) V_x  (carried per row)
// A cancellation guard (||x||^2 < (bb + w^T G w)/64) sends a column to the explicit path
// (x = b0 - V w published, second reduction, GEMV on x): identical results up to rounding.
// scripts/proto_onesync.py checks the algebra against the plain loop.
//
// Layout: rows [rbase, rend) are split into 8-row groups, contiguous per CTA; each CTA owns
// its rows for the whole panel (b, V, Y, Z rows cached in shared memory when they fit), so y
// needs no cross-CTA reduction.  After the sync warps 1..15 stream A for the GEMV while
// warp 0 evaluates the column's scalars; the combine (an 8-lane group per row) then forms
// V(:, j), Y(:, j), Z(:, j) and the next column's b0 and its reduction partials.
// Accumulator sets are indexed by the global column (mod 4) and recycled in-kernel,
// barrier counters alternate between consecutive panel launches: no memsets per panel.
#include <type_traits>

#include "ft_common.cuh"
#include "ft_internal.h"

#include <algorithm>
#include <cstdio>
#include <cstdlib>

#define PT 512        // threads per CTA
#define NW (PT / 32)  // warps per CTA
// GEMV warps: the 12 warps of SM sub-partitions 1..3 (warp w runs on sub-partition w % 4).
// Sub-partition 0 (warps 0, 4, 8, 12) is kept free of the GEMV's load flood, so the control
// warp's shared-memory chain is not queued behind it.
#define NGW (3 * NW / 4)
#define IS_GEMV_WARP(w) (((w) & 3) != 0)
#define GEMV_IDX(w) ((w) - ((w) >> 2) - 1)
// helpers: warps 4, 8, 12 (sub-partition 0, no GEMV) form T(:, j) and the carried Gram while the
// GEMV streams and then stay detached until the next grid sync; the other 13 warps ("workers",
// index wid - wid / 4) run the combine and the column dots, synchronised by named barrier 2
#define IS_HELPER(w) (((w) & 3) == 0 && (w) != 0)
#define NWK (NW - NW / 4 + 1)  // worker warps
#define WKT (32 * NWK)         // worker threads
#define GR 8          // row-group granularity (64 bytes of a column)
#define VS 68         // row stride of the V / Y / Z row caches (doubles; = 4 mod 16: the combine's 8-lane row groups hit distinct banks)
#define RMAX PT       // max rows per CTA
#define NSLOT (PT / 8)  // 8-lane groups per CTA (rows / outputs handled at once)
#ifndef NGLOAD_CG
#define NGLOAD_CG 1
#endif
#if NGLOAD_CG
#define NGLOAD(p) __ldcg(p)
#else
#define NGLOAD(p) (*(p))
#endif
#ifndef GB
// GEMV load batch (double2 of A + b per lane): 6 measured best at C2 (8: +1.5 % panel time, 4: +1 %,
// 12 spills; C3 neutral), profiles/r02/s3b/gemv_loads_ab.txt
#define GB 6
#endif
#define GAMMA (1.0 / 64.0)  // cancellation guard of the one-reduction column (see above)

// accumulator set layout (FT_ACC_STRIDE doubles, each accumulator on its own 256-byte block)
#define ACC_S1 0      // [0, 64)   s1 = V^T b0 (data rows)
#define ACC_SX 64     // [64, 128) V_x^T b0_x (data rows >= c+2)
#define ACC_BB 128    // b0_x . b0_x
#define ACC_EB 129    // e^T b0_x
#define ACC_B0 130    // b0(c+1) (single writer: the row's owner)
#define ACC_FNRM 131  // explicit path: ||x||^2
#define ACC_FEX 132   //                e^T x
#define ACC_FAL 133   //                alpha = b(c+1) (single writer)
#define ACC_FVX 136   // [136, 200)     V^T x
static_assert(ACC_FVX + FT_NBMAX <= FT_ACC_STRIDE, "accumulator set too small");

enum { SC_TAU, SC_BETA, SC_SCALE, SC_ALPHA, SC_VCHK, SC_Q, SC_XX, SC_FB };

struct PanelSmem {
    double Ts[FT_NBMAX][FT_NBMAX + 1];  // Ts[a][b] = T(a, b)
    double Km[FT_NBMAX][FT_NBMAX + 1];  // K = Gp T^T, Gp = Gram of V over rows >= c+1 (see tcol_gram)
    double ku[FT_NBMAX], kst[FT_NBMAX]; // T V(c+1,:)^T, T t (scratch of the K update)
    double s1[FT_NBMAX], w[FT_NBMAX], t[FT_NBMAX], ep[FT_NBMAX];  // ep: e^T V over rows >= c+1
    double vr1[FT_NBMAX + 1];           // V(c+1, 0:j)
    double scal[16];                    // SC_*
    double dsum[2 * FT_NBMAX + 4];      // deterministic mode: the reduced column dots (det_sum)
    double acol[RMAX];                  // A(row, c) of the own rows
    double anext[RMAX];                 // A(row, c+1)
    double b0[RMAX];                    // b0 of the current column
    double bmA[RMAX];                   // b0 masked to the data rows
    double bmX[RMAX];                   // b0 (or x) masked to the data rows >= c+2
    double rref[RMAX];                  // verify: r(row) - Fr(row) of the own rows (loaded in the prologue)
    double2 red[PT];                    // GEMV partials  (y pairs)
    double2 rsr[PT];                    // GEMV partials  (row sums, verify pass)
    unsigned long long drift;           // max fault-free |D_r| of the CTA's rows (reduced once per panel)
    // followed (dynamic part) by the CTA's rows of V, Y and Z when they fit: [R][VS] each
};

size_t ft_panel_smem_bytes() { return sizeof(PanelSmem); }

// timing probes (debug hook): CTA 0's timestamps at dbg[j*16 + slot]; the max over CTAs of
// the cycles since the CTA's previous probe at dbg[1024 + j*16 + slot]
#define PROBE(slot)                                                                   \
    do {                                                                              \
        if (p.dbg && tid == 0 && j < 64) {                                            \
            const long long now_ = clock64();                                         \
            if (bid == 0) p.dbg[j * 16 + (slot)] = now_;                       \
            if ((slot) != 0)                                                          \
                atomicMax(p.dbg + 1024 + j * 16 + (slot), (unsigned long long)(now_ - probe_last)); \
            probe_last = now_;                                                        \
        }                                                                             \
    } while (0)

// DLARFG scalars (reading R1), out of line: one copy of the sqrt / division code
struct Refl {
    double tau, beta, scale;
};
__device__ __forceinline__ Refl dlarfg_scalars(double nrm2, double alpha, bool trivial) {
    Refl r;
    if (nrm2 == 0.0 || trivial) {
        r.tau = 0.0;  // H = I, x left untouched (it is zero)
        r.beta = alpha;
        r.scale = 1.0;
    } else {
        r.beta = -copysign(sqrt(alpha * alpha + nrm2), alpha);  // -sign(alpha) hypot(alpha, ||x||)
        // tau = (beta - alpha) / beta, scale = 1 / (alpha - beta): two independent reciprocals
        // (correctly rounded) instead of two dependent divisions
        const double rb = __drcp_rn(r.beta), rs = __drcp_rn(alpha - r.beta);
        r.tau = (r.beta - alpha) * rb;
        r.scale = rs;
    }
    return r;
}

// 8-lane group sum (lanes g = 0..7 of an aligned group); every lane of the warp must call it
__device__ __forceinline__ double group8_sum(double v) {
    v += __shfl_xor_sync(0xffffffffu, v, 4);
    v += __shfl_xor_sync(0xffffffffu, v, 2);
    v += __shfl_xor_sync(0xffffffffu, v, 1);
    return v;
}

// Partial sums over a in [a0, a1) of w = T^T s1 and k = K s1 for outputs la = lane, lb = lane + 32
// (T, K are zero beyond the current column count).  8 operand rows per batch: all loads of a
// batch are in flight together.
__device__ __forceinline__ void chain_part(const PanelSmem &S, int a0, int a1, int la, int lb, double &wa,
                                           double &wb, double &ka, double &kb) {
    double wa1 = 0.0, wb1 = 0.0, ka1 = 0.0, kb1 = 0.0;
#pragma unroll 1
    for (int b0 = a0; b0 < a1; b0 += 8) {
        double sv[8], ta[8], tb[8], xa[8], xb[8];
#pragma unroll
        for (int u = 0; u < 8; u++) {
            sv[u] = b0 + u < a1 ? S.s1[b0 + u] : 0.0;
            ta[u] = S.Ts[b0 + u][la];
            tb[u] = S.Ts[b0 + u][lb];
            xa[u] = S.Km[la][b0 + u];
            xb[u] = S.Km[lb][b0 + u];
        }
#pragma unroll
        for (int u = 0; u < 8; u += 2) {
            wa += ta[u] * sv[u];
            wb += tb[u] * sv[u];
            ka += xa[u] * sv[u];
            kb += xb[u] * sv[u];
            wa1 += ta[u + 1] * sv[u + 1];
            wb1 += tb[u + 1] * sv[u + 1];
            ka1 += xa[u + 1] * sv[u + 1];
            kb1 += xb[u + 1] * sv[u + 1];
        }
    }
    wa += wa1;
    wb += wb1;
    ka += ka1;
    kb += kb1;
}

// T(:, j) and the carried Gram / e^T V of the next column, from the column's scalars in smem;
// threads t0 = 0..nthr-1 (whole warps) of the calling warps take part.  It runs in helper
// warps concurrently with the GEMV (and on the explicit path after it).  Out of line on purpose:
// inlined into the column loop (as a lambda or a forceinline function) the T(j, j) store was
// addressed from a register not yet defined for the current column (nvcc 12.9, sm_100a).
__device__ __noinline__ void tcol_gram(PanelSmem &S, const int j, const int t0, const int nthr, const bool last) {
    const double tau = S.scal[SC_TAU], scale = S.scal[SC_SCALE];
    // per row c < j of T (an 8-lane group each): st = T(c, :) t, sv = T(c, :) V(c+1, :)^T;
    // T(c, j) = -tau st (DLAHR2 step v)
    const int sl = t0 >> 3, gg = t0 & 7, nsl = nthr >> 3;
    for (int a0 = 0; a0 < j; a0 += nsl) {
        const int c = a0 + sl;
        double st0 = 0.0, st1 = 0.0, sv0 = 0.0, sv1 = 0.0;
        if (c < j)
#pragma unroll
            for (int u = 0; u < FT_NBMAX / 8; u += 2) {
                const int ba = gg + 8 * u, bb2 = ba + 8;
                if (ba < j) {
                    const double tv = S.Ts[c][ba];
                    st0 += tv * S.t[ba];
                    sv0 += tv * S.vr1[ba];
                }
                if (bb2 < j) {
                    const double tv = S.Ts[c][bb2];
                    st1 += tv * S.t[bb2];
                    sv1 += tv * S.vr1[bb2];
                }
            }
        const double st = group8_sum(st0 + st1), sv = group8_sum(sv0 + sv1);
        if (c < j && gg == 0) {
            S.Ts[c][j] = -tau * st;
            S.kst[c] = st;
            S.ku[c] = sv;
        }
    }
    if (t0 == 0) S.Ts[j][j] = tau;
    if (!last) {
        // K = Gp T^T for the next column, without Gp itself.  Gp_new = [Gp - v v^T, g; g^T, sigma]
        // (v = V(c+1, 0:j), g = t - v, sigma = scale^2 ||x||^2) and T_new = [T, tc; 0, tau]
        // (tc = -tau T t) give
        //   K_new(a, c) = K(a, c) - v(a) (T v)(c) + g(a) tc(c)      a, c < j
        //   K_new(a, j) = g(a) tau,   K_new(j, c) = (T g)(c) + sigma tc(c),   K_new(j, j) = sigma tau
        asm volatile("bar.sync 3, %0;\n" ::"r"(nthr) : "memory");
        const double sigma = scale * scale * S.scal[SC_XX];
        const int J1 = j + 1;
        for (int r = t0; r < 2 * J1; r += nthr) {
            const int a = r >> 1, h = r & 1;
            if (a < j) {
                const double va = S.vr1[a], ga = S.t[a] - va;
#pragma unroll 4
                for (int c = h; c < j; c += 2) S.Km[a][c] += -va * S.ku[c] - tau * ga * S.kst[c];
                if (h == 0) S.Km[a][j] = ga * tau;
            } else {
#pragma unroll 4
                for (int c = h; c < j; c += 2) S.Km[j][c] = (S.kst[c] - S.ku[c]) - sigma * tau * S.kst[c];
                if (h == 0) S.Km[j][j] = sigma * tau;
            }
        }
        // e^T V over rows >= c+2
        for (int a = t0; a <= j; a += nthr) S.ep[a] = a < j ? S.ep[a] - S.vr1[a] : S.scal[SC_VCHK] - 1.0;
    }
}

// system-scope flag helpers for the cross-rank exchange (peer memory over NVLink, or the
// other virtual ranks of this launch)
__device__ __forceinline__ unsigned ld_acquire_sys_u32(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_sys_u32(unsigned *p, unsigned v) {
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;\n" ::"l"(p), "r"(v) : "memory");
}

template <int CACHE, bool MG>
__global__ void __launch_bounds__(PT, 1) k_panel(const __grid_constant__ PanelLaunch L) {
    // rank group of this CTA (MG: virtual ranks share the launch; one GPU: a single group)
    const unsigned P = gridDim.x / L.nr;
    const int vr = MG ? (int)(blockIdx.x / P) : 0;
    const PanelParams &p = L.r[vr];
    const int bid = (int)(blockIdx.x - vr * P);
    {
        // the halt flag and, when deferred here, the previous iteration's end-check sums: one round
        // trip, every CTA on the same words (a uniform decision; nobody writes them in this launch)
        const int halted = __ldcg(&p.ctl->halt);
        double e_sr = 0.0, e_sc = 0.0, e_kap = 0.0, e_nf = 0.0, e_thr = 0.0;
        if (p.echeck) {
            e_sr = __ldcg(&p.ctl->sums[2]);
            e_sc = __ldcg(&p.ctl->sums[3]);
            e_kap = __ldcg(p.A + p.n + (int64_t)p.n * p.ldw);
            e_nf = __ldcg(&p.ctl->normF);
            e_thr = __ldcg(&p.ctl->c_thr);
        }
        if (halted) return;
        if (p.echeck) {  // Alg. 3 l.12-13 of iteration echeck_panel (R11/R22), as the fused check
            const double tauS = e_thr * (double)p.n * 2.220446049250313e-16 * e_nf * sqrt((double)p.n);
            const bool bad = p.echeck_policy == FT_POLICY_PAPER
                                 ? not_within(e_sr - e_sc, tauS)
                                 : (not_within(e_sr - e_kap, tauS) || not_within(e_sc - e_kap, tauS));
            if (bad) {
                if (blockIdx.x == 0 && threadIdx.x == 0) {
                    p.ctl->halt_panel = p.echeck_panel;
                    p.ctl->halt_stage = 2;
                    p.ctl->halt_reason = 8;
                    __threadfence();
                    p.ctl->halt = 1;
                }
                return;  // nothing touched: the previous iteration is rolled back
            }
        }
    }
    extern __shared__ __align__(16) unsigned char smem_raw[];
    PanelSmem &S = *reinterpret_cast<PanelSmem *>(smem_raw);

    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int slot = tid >> 3, g = tid & 7;  // 8-lane groups: NSLOT row / output slots
    // wide launches (>= 32 rows per CTA: the GEMV dominates the column) give the GEMV 15 warps,
    // warp 0 forms T(:, j) and the Gram itself, and every warp is a worker
    const bool wide = p.wide != 0;
    const bool gw = wide ? wid != 0 : IS_GEMV_WARP(wid);           // GEMV warp
    const int gidx = wide ? wid - 1 : GEMV_IDX(wid), ngw = wide ? NW - 1 : NGW;
    const bool helper = !wide && IS_HELPER(wid);
    const int nwk = wide ? NW : NWK, wkt = 32 * nwk;
    const int widx = wide ? wid : wid - (wid >> 2), wtid = widx * 32 + lane;  // worker warp / thread index
    // the non-GEMV warps (warp 0 + helpers) as one thread range, for T(:, j) / the Gram
    const int ng_t0 = (wid >> 2) * 32 + lane, ng_n = wide ? 32 : 128;
    const int g0 = (int)((long long)bid * p.ngroups / P);
    const int g1 = (int)((long long)(bid + 1) * p.ngroups / P);
    const int r0 = p.rbase + GR * g0, r1 = p.rbase + GR * g1;
    const int R = r1 - r0, R2 = R >> 1;
    const int n = p.n, ihi = p.ihi, k = p.k, ib = p.ib;
    const int64_t ldw = p.ldw;
    double *__restrict__ A = p.A;
    double *__restrict__ Apan = p.Apan;  // panel columns (== A on one GPU)
    double *__restrict__ V = p.V;
    double *__restrict__ Y = p.Y;

    // own rows of V, Y and Z: [rl][jp] in shared memory (V, Y write-through to global) when
    // they fit, else the global arrays (Z: p.Z)
    // CACHE 2: V, Z, Y rows in smem; 1: V, Z in smem, Y global; 0: all global
    constexpr bool VC = CACHE >= 1, YC = CACHE == 2;
    double *dyn = reinterpret_cast<double *>(smem_raw + sizeof(PanelSmem));
    double *Vl = VC ? dyn : V + r0;
    double *Zl = VC ? dyn + (int64_t)VS * R : p.Z + r0;
    double *Yl = YC ? dyn + (int64_t)2 * VS * R : Y + r0;
    // the CTA's row slab of the columns [k+2, k+2+ncc) at panel start ([col][R]), mode 2 only
    const int ncc = (CACHE == 2 && !MG) ? p.ncc : 0;
    double *Ac = dyn + (int64_t)3 * VS * R;
    constexpr int64_t XR = VC ? VS : 1;  // row stride of V and Z
    const int64_t XC = VC ? 1 : ldw;     // column stride
    constexpr int64_t YR = YC ? VS : 1;  // of Y
    const int64_t YCS = YC ? 1 : ldw;

    // GEMV partial layout: R2p lanes per column, a power of two when <= 32 so the lanes of
    // one row pair are shuffle-reducible inside a warp
    int R2p = R2;
    if (R2 <= 32) {
        R2p = 1;
        while (R2p < R2) R2p *= 2;
    }
    const int ncl = (ngw * 32) / R2p;
    const int npart = R2p <= 32 ? ngw : ncl;  // partials per row pair
    // stride of the partials in S.red / S.rsr: R2p + 1 (odd) when a warp's R2p lanes write one
    // partial each, so the combine's 8 lanes of a row read 8 partials from distinct banks
    const int RSt = R2p <= 32 ? R2p + 1 : R2p;

    auto is_data = [&](int row) { return row >= k + 1 && row < ihi; };
    // fused Y_top: the rows 0..k above the panel take part in the GEMV, Y, Z and b0 (their b0 is
    // the M-part of DGEHRD), never in the column dots, V or the reflectors
    const bool ytop = p.ytop != 0;
    auto is_top = [&](int row) { return ytop && row <= k; };
    auto is_valid = [&](int row) { return (row >= k + 1 && row < ihi) || (p.abft && row == n) || (ytop && row <= k); };

    // ---- CTA-parallel building blocks of the column chain --------------------------------
    // row dot of row rl (an 8-lane group per row): sum_{jp < J} X(rl, jp) z[jp], J <= 64.
    auto rowdot = [&](const double *X, int rl, const double *z, int J) -> double {
        double s0 = 0.0, s1 = 0.0;
        if (rl < R) {
            const double *x = X + rl * XR;
#pragma unroll
            for (int u = 0; u < FT_NBMAX / 8; u += 2) {
                const int ja = g + 8 * u, jb = ja + 8;
                if (ja < J) s0 += x[ja * XC] * z[ja];
                if (jb < J) s1 += x[jb * XC] * z[jb];
            }
        }
        return group8_sum(s0 + s1);
    };
    // column dots over the own rows of V, CTA partials added into the accumulators:
    //   o < JA:            sum_rl V(rl, o) zA[rl]        -> acc[oA + o]
    //   JA <= o < JA + JB: sum_rl V(rl, o - JA) zB[rl]   -> acc[oB + o - JA]
    //   then zB.zB -> acc[oE], sum zB -> acc[oE + 1]
    // An aligned group of LPO lanes per output (4..32, ~2 rows per lane), lanes stride the
    // rows, shuffle tree inside the warp; the group leader adds the CTA partial.
    // a CTA partial of accumulator dst of set acc: FP64 atomic, or (deterministic mode) a store into
    // the CTA's own slot, summed in a fixed order after the grid barrier (det_sum)
    auto acc_add = [&](double *acc, int dst, double s) {
        if (p.dpart)
            p.dpart[((acc - p.acc) / FT_ACC_SET_DOUBLES * FT_ACC_STRIDE + dst) * FT_DPMAX + bid] = s;
        else
            atomicAdd(acc + dst * FT_ACC_PAD, s);
    };
    auto dset = [&](const double *acc) -> const double * {
        return p.dpart + (acc - p.acc) / FT_ACC_SET_DOUBLES * FT_ACC_STRIDE * FT_DPMAX;
    };
    auto coldot_add = [&](const double *zA, int JA, const double *zB, int JB, double *acc, int oA, int oB,
                          int oE) {
        const int NO = JA + JB + 2;
        if (R <= 32) {
            // small row blocks: one worker lane per output, a plain loop over the rows (two
            // chains), no shuffles
            if (helper) return;
            for (int o = wtid; o < NO; o += wkt) {
                const bool ua = o < JA;
                const double *zr = ua ? zA : zB;
                const int col = ua ? o : o - JA;
                const int kind = o < JA + JB ? 0 : (o == JA + JB ? 1 : 2);
                double s0 = 0.0, s1 = 0.0;
                if (kind == 0) {
                    const double *vc = Vl + col * XC;
                    int rl = 0;
#pragma unroll 4
                    for (; rl + 1 < R; rl += 2) {
                        s0 += vc[rl * XR] * zr[rl];
                        s1 += vc[(rl + 1) * XR] * zr[rl + 1];
                    }
                    if (rl < R) s0 += vc[rl * XR] * zr[rl];
                } else {
#pragma unroll 4
                    for (int rl = 0; rl < R; rl++) {
                        const double z = zr[rl];
                        if (kind == 1) s0 += z * z;
                        else s0 += z;
                    }
                }
                if (!(p.dbg_mode & 4)) {
                    const int dst = o < JA ? oA + o : (o < JA + JB ? oB + o - JA : oE + (o - JA - JB));
                    acc_add(acc, dst, s0 + s1);
                }
            }
            return;
        }
        int LPO = 4;
        while (LPO < 32 && 2 * LPO < R && (2 * LPO) * NO <= wkt) LPO *= 2;
        if (helper) return;
        // output blocks of wkt / LPO (two when 4 lanes per output do not cover NO <= 128)
#pragma unroll 1
        for (int ob = 0; ob < NO; ob += wkt / LPO) {
            const int o = ob + wtid / LPO, gl = wtid & (LPO - 1);
            if (ob + (widx * 32) / LPO >= NO) break;  // warp without outputs (warp-uniform)
            double s = 0.0;
            if (o < NO) {
                const bool ua = o < JA;
                const double *zr = ua ? zA : zB;
                const int col = ua ? o : o - JA;
                const int kind = o < JA + JB ? 0 : (o == JA + JB ? 1 : 2);
                double s1 = 0.0;
#pragma unroll 1
                for (int rb = gl; rb < R; rb += 4 * LPO) {
#pragma unroll
                    for (int u = 0; u < 4; u++) {
                        const int rl = rb + u * LPO;
                        if (rl < R) {
                            const double z = zr[rl];
                            const double t = (kind == 0 ? Vl[rl * XR + col * XC] : (kind == 1 ? z : 1.0)) * z;
                            if (u & 1) s1 += t;
                            else s += t;
                        }
                    }
                }
                s += s1;
            }
#pragma unroll
            for (int off = 16; off > 0; off >>= 1)
                if (off < LPO) s += __shfl_xor_sync(0xffffffffu, s, off);
            if (o < NO && gl == 0 && !(p.dbg_mode & 4)) {
                const int dst = o < JA ? oA + o : (o < JA + JB ? oB + o - JA : oE + (o - JA - JB));
                acc_add(acc, dst, s);
            }
        }
    };
    // grid barrier: thread 0 arrives (release, cumulative over the CTA's writes ordered by the
    // bar.sync) and polls (acquire); `after` runs in warp 0 right after the poll succeeds, so
    // the control loads it issues are at the head of the SM's memory queue (ahead of the GEMV)
    auto grid_sync = [&](unsigned &epoch, auto after) {
        __syncthreads();
        if (wid == 0) {
            if (lane == 0 && !(p.dbg_mode & 1)) {
                epoch += 1;
                const unsigned target = epoch * P;
                red_release_add_u32(p.bar, 1u);
                while (ld_acquire_u32(p.bar) < target) {
                }
            }
            __syncwarp();
            after();
        }
        __syncthreads();
    };

    unsigned epoch = 0;
    long long probe_last = 0;
    int j = 0;  // (PROBE)
    if (p.dbg && bid == 0 && tid == 0) p.dbg[3072] = clock64();  // kernel entry (CTA 0): prologue = dbg[0] - this
    // ======================= the trailing GEMV (warps with IS_GEMV_WARP) =========================
    // partials of A(rows, c+2:cend) bv(c+2:cend) (and of the row sums when vfy) into S.red / S.rsr
    auto gemv = [&](const double *bv, int c, bool vfy) {
        const int gt = gidx * 32 + lane;
        const int rp = gt % R2p, cl = gt / R2p;
        const bool gemv_on = rp < R2 && cl < ncl;
        const double2 *__restrict__ A2 = reinterpret_cast<const double2 *>(A + r0);
        const int64_t ldw2 = ldw >> 1;
        const int cend = vfy ? n : ihi;
        double2 ya = make_double2(0.0, 0.0), rs = make_double2(0.0, 0.0);
        if (MG && gemv_on && !(p.dbg_mode & 2)) {
            // virtual columns: [0, nA) the panel columns c+2.. (owner only, from Apan), then
            // the local trailing columns lcol0.. (global index J(l) selects the operand)
            const int nA = (p.owner && p.e > c + 2) ? p.e - (c + 2) : 0;
            const int nv = nA + (p.lcol1 - p.lcol0);
            const double2 *__restrict__ Ap2 = reinterpret_cast<const double2 *>(Apan + r0);
#pragma unroll 1
            for (int v0 = cl; v0 < nv; v0 += GB * ncl) {
                double2 a[GB];
                double xv[GB];
#pragma unroll
                for (int u = 0; u < GB; u++) {
                    const int v = v0 + u * ncl;
                    a[u] = make_double2(0.0, 0.0);
                    xv[u] = 0.0;
                    if (v < nA) {
                        const int q = c + 2 + v;
                        a[u] = Ap2[(int64_t)q * ldw2 + rp];
                        xv[u] = bv[q];
                    } else if (v < nv) {
                        const int l = p.lcol0 + v - nA;
                        const int J = (l / p.cbnb) * p.cbnb * p.G + p.rank * p.cbnb + l % p.cbnb;
                        a[u] = A2[(int64_t)l * ldw2 + rp];
                        xv[u] = J >= c + 2 ? bv[J] : 0.0;  // column c+1 = e is the unit term
                    }
                }
#pragma unroll
                for (int u = 0; u < GB; u++) {
                    ya.x += a[u].x * xv[u];
                    ya.y += a[u].y * xv[u];
                }
            }
        } else if (gemv_on && !(p.dbg_mode & 2)) {
            // bv is read with plain (L1-allocating) loads: the acquire at the grid barrier
            // invalidated this SM's L1 before the trailing bar.sync released us.
            // Columns [k+2, k+2+ncc) come from the CTA's shared-memory copy of its row slab
            // (loaded once per panel), the rest from L2 / HBM.
            auto run = [&](const double2 *__restrict__ base, int64_t cs2, int coff, int cbeg, int cstop, auto glb) {
                // glb: the operand streams from L2 / HBM -- L2-only loads (ld.global.cg, as the wide kernel)
                auto ld = [&](const double2 *ptr) { return decltype(glb)::value ? NGLOAD(ptr) : *ptr; };
                int col = cbeg + cl;
#pragma unroll 1
                for (; col + (GB - 1) * ncl < cstop; col += GB * ncl) {
                    double2 a[GB];
                    double v[GB];
#pragma unroll
                    for (int u = 0; u < GB; u++) {
                        const int q = col + u * ncl;
                        a[u] = ld(base + (int64_t)(q - coff) * cs2 + rp);
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
                if (col < cstop) {  // ragged tail: one predicated batch (all loads in flight together)
                    double2 a[GB];
                    double v[GB];
#pragma unroll
                    for (int u = 0; u < GB; u++) {
                        const int q = col + u * ncl;
                        a[u] = q < cstop ? ld(base + (int64_t)(q - coff) * cs2 + rp) : make_double2(0.0, 0.0);
                        v[u] = q < cstop ? bv[q] : 0.0;
                    }
#pragma unroll
                    for (int u = 0; u < GB; u++) {
                        ya.x += a[u].x * v[u];
                        ya.y += a[u].y * v[u];
                        rs.x += a[u].x;
                        rs.y += a[u].y;
                    }
                }
            };
            const int csplit = min(cend, k + 2 + ncc);
            if (c + 2 < csplit)
                run(reinterpret_cast<const double2 *>(Ac), R2, k + 2, c + 2, csplit, std::integral_constant<bool, false>());
            const int cbeg = max(c + 2, csplit);
            if (cbeg < cend) run(A2, ldw2, 0, cbeg, cend, std::integral_constant<bool, true>());
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
                S.red[gidx * RSt + lane] = ya;
                if (vfy) S.rsr[gidx * RSt + lane] = rs;
            }
        } else if (cl < ncl) {
            S.red[cl * RSt + rp] = ya;
            if (vfy) S.rsr[cl * RSt + rp] = rs;
        }
    };

#pragma unroll 1
    for (int i = tid; i < FT_NBMAX * (FT_NBMAX + 1); i += PT) {
        (&S.Ts[0][0])[i] = 0.0;
        (&S.Km[0][0])[i] = 0.0;
    }
    if (ncc > 0) {
        // the row slab of columns [k+2, k+2+ncc) into shared memory: at panel start they hold
        // A0, and column c's GEMV reads only columns >= c+2, which this panel has not written yet.
        // Issued first: the checkpoint and column-k loads below overlap its flight
        const int R2c = R >> 1;
        for (int x = tid; x < ncc * R2c; x += PT) {
            const int cc = x / R2c, rq = x - cc * R2c;
            cp_async16(Ac + (int64_t)cc * R + 2 * rq, A + (r0 + 2 * rq) + (int64_t)(k + 2 + cc) * ldw, 16);
        }
        cp_async_commit();
    }
    if (p.ckpt) {
        // diskless checkpoint of the panel columns, r, c, kappa, Qr, Qc, Fr, taken
        // before anything is modified: own rows by their owner, the rest grid-strided; all of it
        // precedes this CTA's first arrival
        // (every loop issues its loads before its stores: one round trip per batch, not per word)
        const int rend = p.abft ? n + 1 : ihi;
        // r, Qr, Qc, Fr and the checksum row c, grid-strided: loaded here, in flight with the first
        // batch of panel columns, stored after it (the owner of row n rewrites c(k:e) only after
        // the first grid sync, which every copy precedes)
        const int gstride = (int)P * PT, gi = bid * PT + tid;
        // interleaved over the CTAs (entry bid + P * tid), so CTAs 0..4 carry no extra copies
        const int vi = bid + (int)P * tid;
        double vr = 0.0, vq = 0.0, vc = 0.0, vf = 0.0, vk = 0.0;
        if (vi <= n) {
            vr = p.rcol[vi];
            vq = p.Qr[vi];
            vc = p.Qc[vi];
            vf = p.Fr[vi];
            vk = A[n + (int64_t)vi * ldw];
        }
#pragma unroll 1
        for (int x0 = tid; x0 < R * ib; x0 += 4 * PT) {
            double v[4];
#pragma unroll
            for (int u = 0; u < 4; u++) {
                const int x = x0 + u * PT, rl = x % R, jj = x / R, row = r0 + rl;
                v[u] = (x < R * ib && row < rend) ? Apan[row + (int64_t)(k + jj) * ldw] : 0.0;
            }
#pragma unroll
            for (int u = 0; u < 4; u++) {
                const int x = x0 + u * PT, rl = x % R, jj = x / R, row = r0 + rl;
                if (x < R * ib && row < rend) p.ckpt[row + (int64_t)jj * ldw] = v[u];
            }
        }
#pragma unroll 1
        for (int x0 = gi; x0 < p.rbase * ib; x0 += 4 * gstride) {  // rows above the panel
            double v[4];
#pragma unroll
            for (int u = 0; u < 4; u++) {
                const int x = x0 + u * gstride;
                v[u] = x < p.rbase * ib ? Apan[x % p.rbase + (int64_t)(k + x / p.rbase) * ldw] : 0.0;
            }
#pragma unroll
            for (int u = 0; u < 4; u++) {
                const int x = x0 + u * gstride;
                if (x < p.rbase * ib) p.ckpt[x % p.rbase + (int64_t)(x / p.rbase) * ldw] = v[u];
            }
        }
        if (vi <= n) {
            p.ck_r[vi] = vr;
            p.ck_q[vi] = vq;
            p.ck_q[ldw + vi] = vc;
            p.ck_q[2 * ldw + vi] = vf;
            p.ck_c[vi] = vk;
        }
        for (int i = gi + gstride; i <= n; i += gstride) {  // n >= P * PT only (entries past the first P * PT)
            const double wr = p.rcol[i], wq = p.Qr[i], wc = p.Qc[i], wf = p.Fr[i], wk = A[n + (int64_t)i * ldw];
            p.ck_r[i] = wr;
            p.ck_q[i] = wq;
            p.ck_q[ldw + i] = wc;
            p.ck_q[2 * ldw + i] = wf;
            p.ck_c[i] = wk;
        }
    }
    {
        // column k: b0 = A(:, k); publish its x part (rows >= k+2) and b0(k+1)
        double *acc0 = p.acc + (k & 3) * FT_ACC_SET_DOUBLES;
        double *bv0 = p.bvec + (int64_t)(k & 1) * ldw;
        for (int rl = tid; rl < R; rl += PT) {
            const int row = r0 + rl;
            const double b = is_valid(row) ? Apan[row + (int64_t)k * ldw] : 0.0;
            if (p.verify && (is_data(row) || is_top(row)))  // the D_r reference, in flight with b
                S.rref[rl] = p.rcol[row] - (is_top(row) ? p.Fr[row] : 0.0);
            const bool d = is_data(row), xr = d && row >= k + 2;
            S.acol[rl] = b;
            S.b0[rl] = b;
            S.bmA[rl] = d ? b : 0.0;
            S.bmX[rl] = xr ? b : 0.0;
            if (xr) bv0[row] = b;
            if (row == k + 1 && d) acc0[ACC_B0 * FT_ACC_PAD] = b;
        }
    }
    if (tid < FT_NBMAX) S.ep[tid] = 0.0;
    if (ncc > 0) cp_async_wait<0>();  // the row slab (issued first in the prologue)
    if (tid == 0 && bid == 0) *p.bar_next = 0u;  // the next panel launch's counter
    if (tid == 0) S.drift = 0ull;
    __syncthreads();

    double qc_corner = 0.0;  // corner of the Q checksums: sum of this panel's Qc (CTA 0, thread 0)
    const double c_thr = p.ctl->c_thr;
    const double tau_abs = c_thr * (double)n * 2.220446049250313e-16 * p.ctl->normF;
    // lanes per row in the combine: a whole warp per row for small row blocks
    // lanes per row in the combine (8: 3 shuffle rounds; measured faster than 1 or 32)
    const int lpr = 8;
    const int gl = wtid & (lpr - 1), grp = wtid / lpr, ngrp = wkt / lpr;
    auto gsum = [&](double v) {  // sum over the lpr lanes of a row group
#pragma unroll
        for (int off = 16; off > 0; off >>= 1)
            if (off < lpr) v += __shfl_xor_sync(0xffffffffu, v, off);
        return v;
    };
    // A(row, c+1) of the own rows (thread = row), loaded one column ahead
    // (MG: a trailing column c+1 >= e lives on one rank; it arrives through the exchange)
    // (one GPU: column e is read from A, the panel buffer holds only the panel columns)
    double an_reg = 0.0;
    if (!helper && wtid < R && is_valid(r0 + wtid) && (!MG || k + 1 < p.e))
        an_reg = (k + 1 < p.e ? Apan : A)[(r0 + wtid) + (int64_t)(k + 1) * ldw];

#pragma unroll 1
    for (j = 0; j < ib; j++) {
        const int c = k + j;
        const bool last = j + 1 == ib;
        const bool trivial = c + 2 >= ihi;  // the last reflector of the active block: tau = 0
        double *acc = p.acc + (c & 3) * FT_ACC_SET_DOUBLES;  // accumulator i at acc[i * FT_ACC_PAD]
        const double *bv0 = p.bvec + (int64_t)(c & 1) * ldw;  // b0(c+2:ihi) (GEMV operand)
        double *bvx = p.bvec + (int64_t)(2 + (c & 1)) * ldw;   // x = b(c+2:ihi) (explicit-path operand)
        const bool vfy = (j == 0) && p.verify;
        if (!helper && wtid < R) S.anext[wtid] = an_reg;
        an_reg = 0.0;
        if (!helper && !last && wtid < R && is_valid(r0 + wtid) && (!MG || c + 2 < p.e))
            an_reg = (c + 2 < p.e ? Apan : A)[(r0 + wtid) + (int64_t)(c + 2) * ldw];
        PROBE(0);
        // ---------------- the column's only grid reduction: s1 = V^T b0, sx = V_x^T b0_x,
        // bb = b0_x.b0_x, eb = e^T b0_x (x = data rows >= c+2); b0(c+1) was stored by its owner
        coldot_add(S.bmA, j, S.bmX, j, acc, ACC_S1, ACC_SX, ACC_BB);
        PROBE(1);
        double s1a = 0.0, s1b = 0.0, sxa = 0.0, sxb = 0.0, vra = 0.0, vrb = 0.0, bb = 0.0, eb = 0.0, b0c1 = 0.0;
        grid_sync(epoch, [&]() {
            if (j == 0 && bid == 0 && lane == 0 && p.echeck) {  // every CTA has read the deferred sums
                p.ctl->sums[2] = 0.0;
                p.ctl->sums[3] = 0.0;
            }
            b0c1 = ldcg(acc + ACC_B0 * FT_ACC_PAD);  // single writer
            if (lane < j) vra = ldcg(V + (c + 1) + (int64_t)lane * ldw);
            if (lane + 32 < j) vrb = ldcg(V + (c + 1) + (int64_t)(lane + 32) * ldw);
            if (p.dpart) return;
            bb = ldcg(acc + ACC_BB * FT_ACC_PAD);
            eb = ldcg(acc + ACC_EB * FT_ACC_PAD);
            if (lane < j) {
                s1a = ldcg(acc + (ACC_S1 + lane) * FT_ACC_PAD);
                sxa = ldcg(acc + (ACC_SX + lane) * FT_ACC_PAD);
            }
            if (lane + 32 < j) {
                s1b = ldcg(acc + (ACC_S1 + lane + 32) * FT_ACC_PAD);
                sxb = ldcg(acc + (ACC_SX + lane + 32) * FT_ACC_PAD);
            }
        });
        if (p.dpart) {  // deterministic mode: s1, sx, bb, eb from the CTA partials in a fixed order
            det_sum(dset(acc), (int)P, ACC_S1, j, ACC_SX, j, ACC_BB, 2, S.dsum);
            __syncthreads();
            if (wid == 0) {
                s1a = lane < j ? S.dsum[lane] : 0.0;
                s1b = lane + 32 < j ? S.dsum[lane + 32] : 0.0;
                sxa = lane < j ? S.dsum[j + lane] : 0.0;
                sxb = lane + 32 < j ? S.dsum[j + lane + 32] : 0.0;
                bb = S.dsum[2 * j];
                eb = S.dsum[2 * j + 1];
            }
        }
        PROBE(2);
        if (gw) {
            // speculative: y = A(:, c+1) + scale (A(:, c+2:) b0_x - Z w); MG takes the explicit path
            if (!MG) gemv(bv0, c, vfy);
        } else if (wid == 0) {
            // ======================= control warp: the column's scalars from the reduction =======
            //   w = T^T s1,  G w = Gp w - V(c+1,:)^T q  (G = V_x^T V_x),  q = V(c+1,:) w
            //   ||x||^2 = bb - 2 w.sx + w.Gp w - q^2,  alpha = b0(c+1) - q,  e^T x = eb - ep.w + q
            //   t = V^T v = V(c+1,:)^T + scale (sx - G w)
            // (lane o holds outputs o and o + 32; operand loads are issued 8 rows at a time)
            const int la = lane, lb = lane + 32;
            if (la < j) {
                S.s1[la] = s1a;
                S.vr1[la] = vra;
            }
            if (lb < j) {
                S.s1[lb] = s1b;
                S.vr1[lb] = vrb;
            }
            __syncwarp();
            PROBE(10);
            // w = T^T s1 and k = K s1 (K = Gp T^T: G w = k - V(c+1,:)^T q).  (Splitting this pass
            // over warp 0 and the helpers was measured slower: the chunk is latency-bound.)
            double wa0 = 0.0, wb0 = 0.0, ka0 = 0.0, kb0 = 0.0;
            chain_part(S, 0, j, la, lb, wa0, wb0, ka0, kb0);
            const double wa1 = 0.0, wb1 = 0.0, ka1 = 0.0, kb1 = 0.0;
            const double wa = la < j ? wa0 + wa1 : 0.0, wb = lb < j ? wb0 + wb1 : 0.0;
            const double gpa = ka0 + ka1, gpb = kb0 + kb1;  // (Gp w)(o)
            S.w[la] = wa;
            S.w[lb] = wb;
            PROBE(11);
            const double epa = la < j ? S.ep[la] : 0.0, epb = lb < j ? S.ep[lb] : 0.0;
            double q = vra * wa + vrb * wb, sw = sxa * wa + sxb * wb, ew = epa * wa + epb * wb;
            double wgw = wa * gpa + wb * gpb;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                q += __shfl_xor_sync(0xffffffffu, q, o);
                sw += __shfl_xor_sync(0xffffffffu, sw, o);
                ew += __shfl_xor_sync(0xffffffffu, ew, o);
                wgw += __shfl_xor_sync(0xffffffffu, wgw, o);
            }
            wgw -= q * q;  // w^T G w
            PROBE(12);
            const double xx = bb - 2.0 * sw + wgw;
            const double alpha = b0c1 - q;
            const double ex = trivial ? 0.0 : eb - ew + q;
            // cancellation guard: the expansion loses ~log2((bb + wGw) / xx) bits; below 1/64
            // the column takes the explicit two-reduction path (uniform: every CTA sees the same
            // sums).  MG: always explicit (the ranks' sums differ in rounding, the path must not)
            const bool fast = !MG && !(p.dbg_mode & 8) && (trivial || xx >= GAMMA * (bb + wgw));
            if (fast) {
                const Refl rf = dlarfg_scalars(xx, alpha, trivial);
                if (la < j) S.t[la] = vra + (trivial ? 0.0 : rf.scale * (sxa - (gpa - vra * q)));
                if (lb < j) S.t[lb] = vrb + (trivial ? 0.0 : rf.scale * (sxb - (gpb - vrb * q)));
                if (lane == 0) {
                    S.scal[SC_TAU] = rf.tau;
                    S.scal[SC_BETA] = rf.beta;
                    S.scal[SC_SCALE] = rf.scale;
                    S.scal[SC_ALPHA] = alpha;
                    S.scal[SC_VCHK] = 1.0 + rf.scale * ex;
                    S.scal[SC_XX] = trivial ? 0.0 : xx;
                }
            }
            if (lane == 0) {
                S.scal[SC_Q] = q;
                S.scal[SC_FB] = fast ? 0.0 : 1.0;
            }
            PROBE(9);
            __syncwarp();  // bar.arrive is .aligned: the whole warp, converged, after lane 0's stores
            if (!wide) asm volatile("bar.arrive 1, 128;\n" ::: "memory");  // the scalars are in smem: helpers go
            else if (fast && !(p.dbg_mode & 16)) tcol_gram(S, j, lane, 32, last);
        } else {
            // helpers (warps 4, 8, 12: sub-partition 0, no GEMV): T(:, j) and the carried Gram
            // while the GEMV streams (skipped on the explicit path: done after its second sync)
            __syncwarp();
            asm volatile("bar.sync 1, 128;\n" ::: "memory");
            if (S.scal[SC_FB] == 0.0 && !MG && !(p.dbg_mode & 16)) tcol_gram(S, j, ((wid >> 2) - 1) * 32 + lane, 96, last);
        }
        if (wide) {
            __syncthreads();
        } else if (!helper) {  // workers: GEMV partials, the column's scalars
            __syncwarp();
            asm volatile("bar.sync 2, %0;\n" ::"n"(WKT) : "memory");
        }
        PROBE(3);
        const bool fb = S.scal[SC_FB] != 0.0;  // grid-uniform
        // helpers are done with this column unless the explicit path, MG or the ablation needs them
        if (helper && !fb && !MG && !(p.dbg_mode & 16)) continue;
        if (fb) {
            // ---- explicit path: x = b0 - V w of the own rows, second reduction, GEMV on x
#pragma unroll 1
            for (int base = 0; base < R; base += NSLOT) {
                if (base + 4 * wid >= R) break;
                const int rl = base + slot;
                const double vw = rowdot(Vl, rl, S.w, j);
                if (rl < R && g == 0) {
                    const int row = r0 + rl;
                    const double x = S.b0[rl] - vw;
                    const bool xr = is_data(row) && row >= c + 2;
                    S.bmX[rl] = xr ? x : 0.0;
                    if (xr) bvx[row] = x;
                    if (row == c + 1 && is_data(row)) acc[ACC_FAL * FT_ACC_PAD] = x;
                }
            }
            __syncthreads();
            coldot_add(nullptr, 0, S.bmX, j, acc, 0, ACC_FVX, ACC_FNRM);
            double fnrm = 0.0, fex = 0.0, fal = 0.0, fva = 0.0, fvb = 0.0;
            grid_sync(epoch, [&]() {
                fal = ldcg(acc + ACC_FAL * FT_ACC_PAD);  // single writer
                if (p.dpart) return;
                fnrm = ldcg(acc + ACC_FNRM * FT_ACC_PAD);
                fex = ldcg(acc + ACC_FEX * FT_ACC_PAD);
                if (lane < j) fva = ldcg(acc + (ACC_FVX + lane) * FT_ACC_PAD);
                if (lane + 32 < j) fvb = ldcg(acc + (ACC_FVX + lane + 32) * FT_ACC_PAD);
            });
            if (p.dpart) {  // deterministic mode
                det_sum(dset(acc), (int)P, ACC_FVX, j, ACC_FNRM, 2, 0, 0, S.dsum);
                __syncthreads();
                if (wid == 0) {
                    fva = lane < j ? S.dsum[lane] : 0.0;
                    fvb = lane + 32 < j ? S.dsum[lane + 32] : 0.0;
                    fnrm = S.dsum[j];
                    fex = S.dsum[j + 1];
                }
            }
            if (gw) {
                gemv(bvx, c, false);
            } else if (wid == 0) {
                const Refl rf = dlarfg_scalars(fnrm, fal, trivial);
                if (lane < j) S.t[lane] = S.vr1[lane] + rf.scale * fva;
                if (lane + 32 < j) S.t[lane + 32] = S.vr1[lane + 32] + rf.scale * fvb;
                if (lane == 0) {
                    S.scal[SC_TAU] = rf.tau;
                    S.scal[SC_BETA] = rf.beta;
                    S.scal[SC_SCALE] = rf.scale;
                    S.scal[SC_ALPHA] = fal;
                    S.scal[SC_VCHK] = 1.0 + rf.scale * fex;
                    S.scal[SC_XX] = fnrm;
                }
            }
            __syncthreads();
            if (!gw) tcol_gram(S, j, ng_t0, ng_n, last);  // warp 0 (+ helpers)
        }
        if (MG) {
            // ---- cross-rank exchange of the GEMV partials, CTA by CTA: every rank
            // uses the same row partition, so CTA bid of each rank owns the same rows.  Push
            // (y partial, A(:, c+1) part) of the own rows into every rank's slot, raise the flag,
            // wait for every rank's flag; the combine sums the slots in rank order (identical on
            // every rank).  Slots alternate by column; a rank reaches column c+2's push only
            // after every rank has flagged column c+1, i.e. after it read column c.
            const int sl = c & 1;
            const int l0 = p.lcol0;
            const bool have_an = (c + 1 == p.e) && l0 < p.lcol1 &&
                                 (l0 / p.cbnb) * p.cbnb * p.G + p.rank * p.cbnb + l0 % p.cbnb == p.e;
            for (int rl = tid; rl < R; rl += PT) {
                const int row = r0 + rl, pr = rl >> 1, hi = rl & 1;
                double ys = 0.0;
                for (int q = 0; q < npart; q++) {
                    const double2 u = S.red[q * RSt + pr];
                    ys += hi ? u.y : u.x;
                }
                const double ap = (have_an && is_valid(row)) ? A[row + (int64_t)l0 * ldw] : 0.0;
                const double2 v2 = make_double2(ys, ap);
                for (int gg = 0; gg < p.G; gg++) p.ypeer[gg][((int64_t)sl * p.G + p.rank) * ldw + row] = v2;
            }
            __syncthreads();
            const unsigned seq = p.seq0 + (unsigned)c + 1u;
            if (tid == 0) {
                __threadfence_system();
                for (int gg = 0; gg < p.G; gg++) st_relaxed_sys_u32(p.fpeer[gg] + p.rank * FT_FLAG_STRIDE + bid, seq);
            }
            if (wid == 0 && lane < p.G) {
                unsigned long long t0 = 0ull;
                unsigned polls = 0u;
                while (ld_acquire_sys_u32(p.flags + lane * FT_FLAG_STRIDE + bid) < seq) {
                    peer_spin_guard(t0, polls);
                }
            }
            __syncthreads();
        }
        if ((p.dbg_mode & 16) && !fb) {
            __syncthreads();
            if (!gw) tcol_gram(S, j, ng_t0, ng_n, last);
            __syncthreads();
        }
        PROBE(7);
        // ---------------- combine (lpr lanes per row): with g = the GEMV result,
        //   x = b0 - V w -> V(:, j), reduced column c;   u = scale (g - Z w) (fast) | scale g
        //   y = A(:, c+1) + u,  Y(:, j) = tau (y - Y t);  Z(:, j) = u;  Z -= A(:, c+1) V(c+1, :)
        //   next column's b0 = A(:, c+1) - Y(:, 0:j+1) V(c+1, 0:j+1)^T
        {
            const double tau = S.scal[SC_TAU], beta = S.scal[SC_BETA], scale = S.scal[SC_SCALE];
            const double alpha = S.scal[SC_ALPHA], vchk = S.scal[SC_VCHK], q = S.scal[SC_Q];
            double *accn = p.acc + ((c + 1) & 3) * FT_ACC_SET_DOUBLES;
            double *bvn = p.bvec + (int64_t)((c + 1) & 1) * ldw;
#pragma unroll 1
            for (int base = 0; base < R; base += ngrp) {
                if (helper || base + (widx * 32) / lpr >= R) break;  // warp-uniform: no row for this warp
                const int rl = base + grp;
                const bool on = rl < R && is_valid(r0 + rl);
                const int pr = rl >> 1, hi = rl & 1;
                double gp = 0.0, rsum = 0.0, an_mg = 0.0;
                if (on && MG) {
                    if (gl == 0) {  // exchanged partials, summed in rank order
                        const double2 *yxs = p.yx + (int64_t)(c & 1) * p.G * ldw + (r0 + rl);
                        for (int gg = 0; gg < p.G; gg++) {
                            const double2 u = __ldcg(yxs + (int64_t)gg * ldw);
                            gp += u.x;
                            an_mg += u.y;
                        }
                    }
                } else if (on) {
                    for (int qq = gl; qq < npart; qq += lpr) {
                        const double2 w2 = S.red[qq * RSt + pr];
                        gp += hi ? w2.y : w2.x;
                        if (vfy) {
                            const double2 r2 = S.rsr[qq * RSt + pr];
                            rsum += hi ? r2.y : r2.x;
                        }
                    }
                }
                double zw = 0.0, vw = 0.0, yt = 0.0, yr = 0.0;
                if (on) {
                    const double anl = S.anext[rl];
#pragma unroll 2
                    for (int i = gl; i < j; i += lpr) {
                        const double wi = S.w[i], vri = S.vr1[i], ti = S.t[i];
                        double *zp = Zl + rl * XR + i * XC;
                        const double z = *zp, vv = Vl[rl * XR + i * XC], yv = Yl[rl * YR + i * YCS];
                        zw += z * wi;
                        vw += vv * wi;
                        yt += yv * ti;
                        yr += yv * vri;
                        if (!last) *zp = z - anl * vri;
                    }
                }
                PROBE(14);
                // six group sums, interleaved (independent shuffle chains)
#pragma unroll
                for (int off = 16; off > 0; off >>= 1) {
                    if (off < lpr) {
                        const double a0 = __shfl_xor_sync(0xffffffffu, gp, off);
                        const double a1 = __shfl_xor_sync(0xffffffffu, zw, off);
                        const double a2 = __shfl_xor_sync(0xffffffffu, vw, off);
                        const double a3 = __shfl_xor_sync(0xffffffffu, yt, off);
                        const double a4 = __shfl_xor_sync(0xffffffffu, yr, off);
                        const double a5 = __shfl_xor_sync(0xffffffffu, rsum, off);
                        gp += a0;
                        zw += a1;
                        vw += a2;
                        yt += a3;
                        yr += a4;
                        rsum += a5;
                    }
                }
                PROBE(15);
                if (rl < R && gl == 0) {
                    const int row = r0 + rl;
                    const double an = (MG && c + 1 >= p.e) ? an_mg : S.anext[rl];
                    double b0n = 0.0;
                    if (on) {
                        const double b = S.b0[rl] - vw;  // b = b0 - V T^T V^T b0 (step ii)
                        // V(:, j) and the reduced column c of the own rows (step iii)
                        if (row == n && p.abft) {
                            V[row + (int64_t)j * ldw] = vchk;
                            if (VC) Vl[rl * XR + j * XC] = vchk;
                            Apan[row + (int64_t)c * ldw] = (tau != 0.0) ? b - vchk * (alpha - beta) : b;  // left term (R7)
                        } else {
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
                            if (VC) Vl[rl * XR + j * XC] = vv;
                            Apan[row + (int64_t)c * ldw] = av;
                        }
                        // steps (iv)-(v)
                        const double u = fb ? scale * gp : scale * (gp - (zw - an * q));
                        if (!last) Zl[rl * XR + j * XC] = u;
                        const double yy = tau * (an + u - yt);
                        Y[row + (int64_t)j * ldw] = yy;
                        if (YC) Yl[rl * YR + j * YCS] = yy;
                        b0n = an - yr - yy;
                        if (vfy && (is_data(row) || is_top(row))) {
                            // D_r(row) = r(row) - sum_{col >= k} L(row, col); columns < k are logical zero
                            // for data rows, the frozen finished-H sums Fr for the rows above (area 1)
                            rsum += S.acol[rl] + an;
                            const double d = S.rref[rl] - rsum;
                            if (not_within(d, tau_abs)) {
                                atomicAdd(&p.ctl->nflag, 1);
                            } else if (tau_abs > 0.0) {
                                const double rel = fabs(d) / (tau_abs / c_thr);
                                atomicMax(&S.drift, (unsigned long long)__double_as_longlong(rel));  // smem: one global max per CTA
                            }
                        }
                    } else if (VC) {
                        Vl[rl * XR + j * XC] = 0.0;  // rows outside the panel take no part in the dots
                    }
                    S.acol[rl] = an;
                    S.b0[rl] = b0n;
                    if (!last) {  // publish the next column's b0
                        const bool d = on && is_data(row), xr = d && row >= c + 3;
                        S.bmA[rl] = d ? b0n : 0.0;
                        S.bmX[rl] = xr ? b0n : 0.0;
                        if (xr) bvn[row] = b0n;
                        if (row == c + 2 && d) accn[ACC_B0 * FT_ACC_PAD] = b0n;
                    }
                }
            }
            PROBE(13);
            if (bid == 0 && tid == 0) {
                p.tau[c] = tau;
                if (p.abft) {
                    p.Qc[c] = vchk - 1.0;  // Q column checksum
                    qc_corner += vchk - 1.0;
                }
            }
            // recycle the accumulator set of column c+2 (= that of column c-2): every CTA has
            // finished reading it, and column c+2 adds into it only after two more syncs
            if (bid == 0 && wid == NW - 1)
                for (int i = lane; i < FT_ACC_STRIDE; i += 32)
                    p.acc[((c + 2) & 3) * FT_ACC_SET_DOUBLES + i * FT_ACC_PAD] = 0.0;
            if (wide) {
                __syncthreads();
            } else if (!helper) {  // workers: the next column's b0 and masks are in smem
                __syncwarp();
                asm volatile("bar.sync 2, %0;\n" ::"n"(WKT) : "memory");
            }
        }
        PROBE(8);
    }
    __syncthreads();  // the helpers' last T column
    __syncthreads();
    if (tid == 0 && S.drift) atomicMax(&p.ctl->drift_bits, S.drift);
    // Q row checksums of the new Householder vectors (Fig. 5): own data rows
    if (p.abft)
        for (int rl = tid; rl < R; rl += PT) {
            const int row = r0 + rl;
            if (!is_data(row)) continue;
            double s = 0.0;
            for (int jj = 0; jj < ib; jj++)
                if (row >= k + jj + 2) s += Vl[rl * XR + jj * XC];
            atomicAdd(&p.Qr[row], s);  // one writer per row: a plain Qr + s, without the load round trip
        }
    if (p.precheck_sums) {  // e^T Y, e^T V over the own data rows (pre-update check R15, fused): 8 lanes per sum
        const int l8 = tid & 7;  // 2 ib <= 128 sums over 64 groups; the loop bound is warp-uniform
        for (int base = (tid >> 5) * 4; base < 2 * ib; base += PT / 8) {
            const int oo = base + ((tid >> 3) & 3), jj = oo % ib;
            double s = 0.0;
            if (oo < 2 * ib)
                for (int rl = l8; rl < R; rl += 8)
                    if (is_data(r0 + rl) || is_top(r0 + rl)) s += oo < ib ? Yl[rl * YR + jj * YCS] : Vl[rl * XR + jj * XC];
            s += __shfl_xor_sync(0xffffffffu, s, 1);
            s += __shfl_xor_sync(0xffffffffu, s, 2);
            s += __shfl_xor_sync(0xffffffffu, s, 4);
            if (l8 == 0 && oo < 2 * ib) atomicAdd(oo < ib ? &p.ctl->eY[jj * FT_ESTR] : &p.ctl->eV[jj * FT_ESTR], s);
        }
    }
    if (bid == 0 && tid == 0 && p.abft) atomicAdd(&p.Qc[n], qc_corner);  // single writer: Qc(n) + corner
    // T, max |T| and the T checksum from three different CTAs (every CTA holds T in shared memory),
    // so no CTA carries all three serial tails
    const int P3 = (int)P;
    if (bid == (P3 > 1 ? 1 : 0))
        for (int i = tid; i < ib * ib; i += PT) p.T[i % ib + (i / ib) * FT_NBMAX] = S.Ts[i % ib][i / ib];
    if (p.precheck_sums && bid == (P3 > 2 ? 2 : 0)) {  // max |T| for the pre-update tolerance (R15)
        double tm = 0.0;
        for (int i = tid; i < ib * ib; i += PT) tm = fmax(tm, fabs(S.Ts[i % ib][i / ib]));
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) tm = fmax(tm, __shfl_xor_sync(0xffffffffu, tm, o));
        if (lane == 0) S.red[wid].x = tm;
        __syncthreads();
        if (tid == 0) {
            double m = 0.0;
            for (int w = 0; w < NW; w++) m = fmax(m, S.red[w].x);
            p.ctl->tmax = m;
        }
    }
    if (p.abft && bid == (P3 > 3 ? 3 : 0) && tid < 4 * FT_NBMAX) {  // T checksum (R15 extended to T)
        double ts, tsa;
        t_row_checksum([&](int a, int bb) { return S.Ts[a][bb]; }, tid >> 2, tid & 3, ib, ts, tsa);
        if ((tid & 3) == 0 && (tid >> 2) < ib) p.ctl->tchk[tid >> 2] = ts;
    }
    if (p.dbg && bid == 0) {  // epilogue end (CTA 0): epilogue = this - the last column's end
        __syncthreads();
        if (tid == 0) p.dbg[3073] = clock64();
    }
}

cudaError_t ft_launch_panel_multi(const PanelLaunch &L, int nsm, cudaStream_t s) {
    static int max_smem = 0;
    static unsigned attr = 0;
    const unsigned dbit = ft_dev_bit();
    if (!(attr & dbit)) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        const void *fns[] = {(const void *)k_panel<2, false>, (const void *)k_panel<1, false>,
                             (const void *)k_panel<0, false>, (const void *)k_panel<2, true>,
                             (const void *)k_panel<1, true>, (const void *)k_panel<0, true>};
        for (const void *fn : fns) {
            cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem);
            if (e != cudaSuccess) return e;
        }
        attr |= dbit;
    }
    static int ctas = -1, explicit_path = 0;
    if (ctas < 0) {
        ctas = ft_panel_cta_cap();
        const char *x = getenv("FT_PANEL_EXPLICIT");  // experiment knob: every column on the explicit path
        explicit_path = x ? atoi(x) : 0;
        const char *d = getenv("FT_PANEL_DBG");  // experiment knob: dbg_mode bits for every launch
        if (d) explicit_path |= atoi(d) << 8;
    }
    if (L.nr < 1 || L.nr > FT_MAX_VRANKS) return cudaErrorInvalidValue;
    const bool mg = L.r[0].G > 1;
    int per = nsm / L.nr;  // CTAs per rank group (identical row partition in every group)
    if (ctas > 0 && ctas < per) per = ctas;
    if (per > FT_FLAG_STRIDE) per = FT_FLAG_STRIDE;
    int grid = per < L.r[0].ngroups ? per : L.r[0].ngroups;
    if (grid < 1) grid = 1;
    // rows per CTA (max over CTAs) and whether their V/Y/Z rows fit next to the fixed part
    const int gmax = (L.r[0].ngroups + grid - 1) / grid;
    const int rmax = GR * gmax;
    if (rmax > WKT) return cudaErrorInvalidConfiguration;  // n beyond ~61k rows per GPU
    const size_t fixed = sizeof(PanelSmem);
    const size_t row_bytes = (size_t)VS * rmax * sizeof(double);
    // mode 1 (V, Z rows cached, Y global) is kept for tests only: at the sizes where mode 2 does
    // not fit, the GEMV streams from HBM and needs the L1 that a >200 KB carve-out would take
    int cache = fixed + 3 * row_bytes <= (size_t)max_smem ? 2 : 0;
    if ((L.r[0].dbg_mode & 64) && cache > 1) cache = 1;  // test hooks: force the smaller caching modes
    if (L.r[0].dbg_mode & 128) cache = 0;
    size_t want = fixed + (size_t)(cache == 2 ? 3 : (cache == 1 ? 2 : 0)) * row_bytes;
    // mode 2, one GPU: the rest of shared memory caches the CTAs' row slabs of the first trailing
    // columns for the whole panel (each column's GEMV would otherwise re-read them from L2)
    int ncc = 0;
    if (cache == 2 && !mg) {
        static int ncc_cap = -1;
        if (ncc_cap < 0) {
            const char *e = getenv("FT_PANEL_NCC");  // experiment knob: cap on the cached columns
            ncc_cap = e ? atoi(e) : 1 << 30;
        }
        ncc = (int)(((size_t)max_smem - want) / ((size_t)rmax * sizeof(double)));
        ncc = std::min(ncc, std::min(ncc_cap, L.r[0].n - L.r[0].k - 2));
        if (ncc < 0) ncc = 0;
        want += (size_t)ncc * rmax * sizeof(double);
    }
    // wide single-GPU launches: the two-reduction kernel (ft_panel_wide.cu), see its header
    // (FT_WIDE_MIN_ROWS: the rows-per-CTA threshold of the wide kernel, for A/B runs)
    static const int wide_min = getenv("FT_WIDE_MIN_ROWS") ? atoi(getenv("FT_WIDE_MIN_ROWS")) : 32;
    if (L.nr == 1 && !mg && rmax >= wide_min && !(L.r[0].dbg_mode & (8 | 64 | 128)) && !explicit_path)
        return ft_launch_panel_wide(L, nsm, s);
    PanelLaunch Lx = L;
    for (int i = 0; i < Lx.nr; i++) {
        Lx.r[i].wide = rmax >= 32 ? 1 : 0;
        Lx.r[i].ncc = ncc;
        if (explicit_path) Lx.r[i].dbg_mode |= ((explicit_path & 0xff) ? 8 : 0) | (explicit_path >> 8);
    }
    if (L.r[0].dpart && grid > FT_DPMAX) return cudaErrorInvalidValue;  // deterministic mode: partial slots
    const PanelLaunch *Lp = &Lx;
    void *args[] = {const_cast<PanelLaunch *>(Lp)};
    g_ft_launches++;
    const void *fn = mg ? (cache == 2 ? (const void *)k_panel<2, true>
                                      : (cache == 1 ? (const void *)k_panel<1, true> : (const void *)k_panel<0, true>))
                        : (cache == 2 ? (const void *)k_panel<2, false>
                                      : (cache == 1 ? (const void *)k_panel<1, false> : (const void *)k_panel<0, false>));
    return cudaLaunchCooperativeKernel(fn, dim3(grid * L.nr), dim3(PT), args, want, s);
}

cudaError_t ft_launch_panel(const PanelParams &p, int nsm, cudaStream_t s) {
    PanelLaunch L;
    L.r[0] = p;
    L.nr = 1;
    L.r[0].G = 1;
    if (!L.r[0].Apan) L.r[0].Apan = p.A;
    if (!L.r[0].rcol) L.r[0].rcol = p.A + (int64_t)p.n * p.ldw;
    if (!L.r[0].e) L.r[0].e = p.k + p.ib;
    return ft_launch_panel_multi(L, nsm, s);
}

int ft_panel_group_rows() { return GR; }
// FT_PANEL_CTAS (experiment knob): a cap on the panel grid (0: one CTA per SM); the driver's fused-Y_top
// decision (<= 24 rows per CTA) uses the same effective count
int ft_panel_cta_cap() {
    static int cap = -1;
    if (cap < 0) {
        const char *e = getenv("FT_PANEL_CTAS");
        cap = e ? atoi(e) : 0;
        if (cap < 0) cap = 0;
    }
    return cap;
}
