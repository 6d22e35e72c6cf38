// ft_panel_wide.cu -- the two-reduction DLAHR2 panel kernel, used for WIDE launches (>= 32
// rows per CTA: the trailing GEMV streams from HBM and dominates every column, so the column
// chain's second grid reduction is hidden, while the GEMV wants all 15 warps and the smallest
// shared-memory carve-out).  Narrow launches (the latency-bound regime) use the one-reduction
// kernel of ft_panel.cu.  Same PanelParams, accumulator sets, barrier counters and outputs.
//
// (original header of this kernel)
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
#define NGW NW  // GEMV warps (warp 0, the control warp, joins after its chain work)
// row-group granularity of the CTA row blocks (64 bytes of a column; the driver's ft_panel_group_rows).
// 2-row groups (equal rows per CTA to one double2) measured no faster at C3: the slowest CTAs of a
// column are set by the address position of their rows, not by the +8-row blocks
#ifndef GR
#define GR 8
#endif
#define GR_DRIVER 8
#define VS 65         // shared-memory row stride of the V / Y row caches (doubles)
#define RMAX PT       // max rows per CTA
#define NSLOT (PT / 8)  // 8-lane groups per CTA (rows / outputs handled at once)
// GEMV loads of A: L2 only (ld.global.cg) -- A streams once per column and never hits L1, and
// bypassing L1 measured -1.2 % panel time at C3; evict-first: +3 %; nc.no_allocate: 0
// (profiles/r02/s3b/gemv_loads_ab.txt)
#define GLOAD(p) __ldcg(p)
#ifndef GB
// GEMV load batch (double2 of A + b per lane): 12 streams at 0.9 of the HBM copy bandwidth at C3
// (8: -1.4 % panel time; 16 spills; a software-pipelined 2 x 6 / 2 x 8 batch: +8 %,
// profiles/r02/s3/gemv_batch_ab.txt)
#define GB 12
#endif

// accumulator set layout (FT_ACC_STRIDE doubles): [0,64) s1 = V^T b0 | [64,128) V^T x |
// 128 ||x||^2 | 129 e^T x | 130 alpha
#define ACC_VTB 64
#define ACC_NRM 128
#define ACC_SX 129
#define ACC_ALPHA 130

struct PanelSmemW {
    double Ts[FT_NBMAX][FT_NBMAX + 1];  // Ts[a][b] = T(a, b)
    double vrow[FT_NBMAX];              // V(c, 0:j) of the current column
    double w[FT_NBMAX];                 // T^T s1
    double t[FT_NBMAX];                 // V^T v
    double s1[FT_NBMAX];                // V^T b0 (reduced)
    double scal[8];                     // tau, beta, scale, vchk, alpha
    double dsum[2 * FT_NBMAX + 4];      // deterministic mode: the reduced column dots (det_sum)
    double acol[RMAX];                  // A(row, c) of the own rows
    double anext[RMAX];                 // A(row, c+1)
    double b0[RMAX];                    // b0 (rows), then b
    double bm[RMAX];                    // masked b0 / x for the column dots
    double2 red[PT];                    // GEMV partials  (y pairs)
    double2 rsr[PT];                    // GEMV partials  (row sums, verify pass)
    unsigned long long drift;           // max fault-free |D_r| of the CTA's rows (reduced once per panel)
    // followed (dynamic part) by the CTA's rows of V and Y when they fit: [R][VS] each
};


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

// 8-lane group sum (lanes g = 0..7 of an aligned group); every lane of the warp must call it
__device__ __forceinline__ double group8_sum(double v) {
    v += __shfl_xor_sync(0xffffffffu, v, 4);
    v += __shfl_xor_sync(0xffffffffu, v, 2);
    v += __shfl_xor_sync(0xffffffffu, v, 1);
    return v;
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

template <bool CACHE, bool MG>
__global__ void __launch_bounds__(PT, 1) k_panel_wide(const __grid_constant__ PanelLaunch L) {
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
    PanelSmemW &S = *reinterpret_cast<PanelSmemW *>(smem_raw);

    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int slot = tid >> 3, g = tid & 7;  // 8-lane groups: NSLOT row / output slots
    // row block of this CTA (dbg_mode >> 16: a rotation of the block <-> CTA map, probe experiments)
    const int pbid = (int)((bid + (unsigned)(p.dbg_mode >> 16)) % P);
    const int g0 = (int)((long long)pbid * p.ngroups / P);
    const int g1 = (int)((long long)(pbid + 1) * p.ngroups / P);
    const int r0 = p.rbase + GR * g0, r1 = p.rbase + GR * g1;
    const int R = r1 - r0, R2 = R >> 1;
    const int n = p.n, ihi = p.ihi, k = p.k, ib = p.ib;
    const int64_t ldw = p.ldw;
    double *__restrict__ A = p.A;
    double *__restrict__ Apan = p.Apan;  // panel columns (== A on one GPU)
    double *__restrict__ V = p.V;
    double *__restrict__ Y = p.Y;

    // own rows of V and Y: [rl][jp] in shared memory (write-through to global) when they fit
    double *Vl = CACHE ? reinterpret_cast<double *>(smem_raw + sizeof(PanelSmemW)) : V + r0;
    double *Yl = CACHE ? Vl + (int64_t)VS * R : Y + r0;
    constexpr int64_t XR = CACHE ? VS : 1;  // row stride
    const int64_t XC = CACHE ? 1 : ldw;     // column stride

    // GEMV partial layout: R2p lanes per column, a power of two when <= 32 so the lanes of
    // one row pair are shuffle-reducible inside a warp
    int R2p = R2;
    if (R2 <= 32) {
        R2p = 1;
        while (R2p < R2) R2p *= 2;
    }
    const int ncl = (NGW * 32) / R2p;
    const int npart = R2p <= 32 ? NGW : ncl;  // partials per row pair

    auto is_data = [&](int row) { return row >= k + 1 && row < ihi; };
    // deterministic mode: the partial block of the accumulator set `acc` belongs to
    auto dset = [&](const double *acc) -> const double * {
        return p.dpart + (acc - p.acc) / FT_ACC_SET_DOUBLES * FT_ACC_STRIDE * FT_DPMAX;
    };
    auto is_valid = [&](int row) { return (row >= k + 1 && row < ihi) || (p.abft && row == n); };

    // ---- CTA-parallel building blocks of the column chain --------------------------------
    // row dot of row rl (an 8-lane group per row): sum_{jp < J} X(rl, jp) z[jp], J <= 64.
    // Fully unrolled with predication: all operand loads are in flight at once.
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
    // column dots over the own rows, CTA partial added into the accumulators:
    // out[o] = sum_rl X(rl, o) zr[rl] (o < J); extras: out[J] = zr.zr, out[J+1] = sum zr.
    // An aligned group of LPO lanes per output (4..32: ~2 rows per lane, LPO * outputs <= PT),
    // lanes stride the rows, shuffle tree inside the warp; the group leader adds the CTA
    // partial into the accumulator.  No shared-memory pass, no CTA barrier.
    auto coldot_add = [&](const double *X, const double *zr, int J, bool extras, double *acc, int acc_o0,
                          int acc_extra0) {
        const int NO = J + (extras ? 2 : 0);
        // lanes per output: ~2 rows per lane, at most 32, at most PT / NO (a power of two)
        int LPO = 4;
        while (LPO < 32 && 2 * LPO < R && (2 * LPO) * NO <= PT) LPO *= 2;
        const int o = tid / LPO, gl = tid & (LPO - 1);
        if ((wid * 32) / LPO >= NO) return;  // warp without outputs (warp-uniform)
        double s = 0.0;
        if (o < NO) {
            double s1 = 0.0;
#pragma unroll 1
            for (int rb = gl; rb < R; rb += 4 * LPO) {
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    const int rl = rb + u * LPO;
                    if (rl < R) {
                        const double z = zr[rl];
                        const double t = (o < J ? X[rl * XR + o * XC] : (o == J ? z : 1.0)) * z;
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
            const int dst = o < J ? acc_o0 + o : acc_extra0 + (o - J);
            if (p.dpart)  // deterministic mode: this CTA's partial in its own slot
                p.dpart[((acc - p.acc) / FT_ACC_SET_DOUBLES * FT_ACC_STRIDE + dst) * FT_DPMAX + bid] = s;
            else
                atomicAdd(acc + dst * FT_ACC_PAD, s);
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

#pragma unroll 1
    for (int i = tid; i < FT_NBMAX * (FT_NBMAX + 1); i += PT) (&S.Ts[0][0])[i] = 0.0;
    if (p.ckpt) {
        // diskless checkpoint of the panel columns, r, c, kappa, Qr, Qc, Fr, taken
        // before anything is modified: own rows by their owner, the rest grid-strided; all of it
        // precedes this CTA's first arrival
        // (every loop issues its loads before its stores: one round trip per batch, not per word)
        const int rend = p.abft ? n + 1 : ihi;
#pragma unroll 1
        for (int x0 = tid; x0 < R * ib; x0 += 8 * PT) {
            double v[8];
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int x = x0 + u * PT, rl = x % R, jj = x / R, row = r0 + rl;
                v[u] = (x < R * ib && row < rend) ? Apan[row + (int64_t)(k + jj) * ldw] : 0.0;
            }
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int x = x0 + u * PT, rl = x % R, jj = x / R, row = r0 + rl;
                if (x < R * ib && row < rend) p.ckpt[row + (int64_t)jj * ldw] = v[u];
            }
        }
        const int gstride = (int)P * PT, gi = bid * PT + tid;
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
        // r, Qr, Qc, Fr and the checksum row c, grid-strided: every copy precedes its CTA's first
        // arrival, and the owner of row n rewrites c(k:e) only after that first grid sync
        for (int i = gi; i <= n; i += gstride) {
            const double vr = p.rcol[i], vq = p.Qr[i], vc = p.Qc[i], vf = p.Fr[i], vk = A[n + (int64_t)i * ldw];
            p.ck_r[i] = vr;
            p.ck_q[i] = vq;
            p.ck_q[ldw + i] = vc;
            p.ck_q[2 * ldw + i] = vf;
            p.ck_c[i] = vk;
        }
    }
    for (int rl = tid; rl < R; rl += PT) {
        const int row = r0 + rl;
        S.acol[rl] = is_valid(row) ? Apan[row + (int64_t)k * ldw] : 0.0;
    }
    if (tid == 0 && bid == 0) *p.bar_next = 0u;  // the next panel launch's counter
    if (tid == 0) S.drift = 0ull;
    __syncthreads();

    unsigned epoch = 0;
    long long probe_last = 0;
    double qc_corner = 0.0;  // corner of the Q checksums: sum of this panel's Qc (CTA 0, thread 0)
    const double c_thr = p.ctl->c_thr;
    const double tau_abs = c_thr * (double)n * 2.220446049250313e-16 * p.ctl->normF;

#pragma unroll 1
    for (int j = 0; j < ib; j++) {
        const int c = k + j;
        double *acc = p.acc + (c & 3) * FT_ACC_SET_DOUBLES;  // accumulator i at acc[i * FT_ACC_PAD]
        // A(row, c+1) of the own rows (thread = row): issued now, parked in smem before the GEMV
        double an_reg = 0.0;
        // (MG: a trailing column c+1 >= e lives on one rank; it arrives through the exchange)
        // (one GPU: column e is read from A, the panel buffer holds only the panel columns)
        if (tid < R && is_valid(r0 + tid) && (!MG || c + 1 < p.e))
            an_reg = (c + 1 < p.e ? Apan : A)[(r0 + tid) + (int64_t)(c + 1) * ldw];
        PROBE(0);
        // ---------------- (i) b0 = A(:,c) - Y V(c,:)^T, s1 = V^T b0 ---------------------------
        if (j > 0) {
            // b0 = A(:, c) - Y V(c, :)^T of the own rows was formed by the previous column's
            // step (v) (S.b0 / S.bm): only the column dots remain here
            coldot_add(Vl, S.bm, j, false, acc, 0, 0);
            PROBE(1);
            grid_sync(epoch, [&]() {
                if (p.dpart) return;
                if (lane < j) S.s1[lane] = ldcg(acc + lane * FT_ACC_PAD);
                if (lane + 32 < j) S.s1[lane + 32] = ldcg(acc + (lane + 32) * FT_ACC_PAD);
            });
            if (p.dpart) {  // deterministic mode: fixed-order sums of the CTA partials
                det_sum(dset(acc), (int)P, 0, j, 0, 0, 0, 0, S.s1);
                __syncthreads();
            }
            PROBE(2);
            // w = T^T s1 (an 8-lane group per output)
            {
                double s0 = 0.0, s1 = 0.0;
                if (4 * wid < j) {
                if (slot < j)
#pragma unroll
                    for (int u = 0; u < FT_NBMAX / 8; u += 2) {
                        const int ba = g + 8 * u, bb = ba + 8;
                        if (ba <= slot) s0 += S.Ts[ba][slot] * S.s1[ba];
                        if (bb <= slot) s1 += S.Ts[bb][slot] * S.s1[bb];
                    }
                const double s = group8_sum(s0 + s1);
                if (slot < j && g == 0) S.w[slot] = s;
                }
            }
            __syncthreads();
        }
        // ---------------- (ii) b = b0 - V w; publish x = b(c+2:ihi) for the GEMV, alpha = b(c+1)
        auto publish = [&](int rl, double b) {
            const int row = r0 + rl;
            const bool xrow = is_data(row) && row >= c + 2;
            S.b0[rl] = b;
            S.bm[rl] = xrow ? b : 0.0;
            if (xrow) p.bvec[row] = b;
            if (row == c + 1) acc[ACC_ALPHA * FT_ACC_PAD] = b;  // alpha: a single writer
        };
        if (j > 0) {
#pragma unroll 1
            for (int base = 0; base < R; base += NSLOT) {
                if (base + 4 * wid >= R) break;
                const int rl = base + slot;
                const double vw = rowdot(Vl, rl, S.w, j);
                if (rl < R && g == 0) publish(rl, S.b0[rl] - vw);
            }
        } else {
            for (int rl = tid; rl < R; rl += PT) publish(rl, S.acol[rl]);
        }
        __syncthreads();
        PROBE(3);
        coldot_add(Vl, S.bm, j, true, acc, ACC_VTB, ACC_NRM);
        if (tid < R) S.anext[tid] = an_reg;
        PROBE(4);
        // control scalars of DLARFG, loaded by warp 0 as soon as the barrier opens
        double nrm2 = 0.0, sx = 0.0, alpha = 0.0, vn0 = 0.0, vt0 = 0.0, vn1 = 0.0, vt1 = 0.0;
        grid_sync(epoch, [&]() {
            if (j == 0 && bid == 0 && lane == 0 && p.echeck) {  // every CTA has read the deferred sums
                p.ctl->sums[2] = 0.0;
                p.ctl->sums[3] = 0.0;
            }
            alpha = ldcg(acc + ACC_ALPHA * FT_ACC_PAD);  // single writer
            if (lane < j) vn0 = ldcg(V + (c + 1) + (int64_t)lane * ldw);
            if (lane + 32 < j) vn1 = ldcg(V + (c + 1) + (int64_t)(lane + 32) * ldw);
            if (p.dpart) return;
            nrm2 = ldcg(acc + ACC_NRM * FT_ACC_PAD);
            sx = ldcg(acc + ACC_SX * FT_ACC_PAD);
            if (lane < j) vt0 = ldcg(acc + (ACC_VTB + lane) * FT_ACC_PAD);
            if (lane + 32 < j) vt1 = ldcg(acc + (ACC_VTB + lane + 32) * FT_ACC_PAD);
        });
        if (p.dpart) {  // deterministic mode: V^T x, ||x||^2, e^T x from the CTA partials in a fixed order
            det_sum(dset(acc), (int)P, ACC_VTB, j, ACC_NRM, 2, 0, 0, S.dsum);
            __syncthreads();
            if (wid == 0) {
                vt0 = lane < j ? S.dsum[lane] : 0.0;
                vt1 = lane + 32 < j ? S.dsum[lane + 32] : 0.0;
                nrm2 = S.dsum[j];
                sx = S.dsum[j + 1];
            }
        }
        PROBE(5);
        unsigned long long gt_start = 0;
        if (p.dbg && tid == 0 && j == 8) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt_start));
        if (wid == 0) {
            // ======================= control warp: (iii) DLARFG (R1), V(:, j) ================
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
            PROBE(9);
            // V(:, j) and the reduced column c of the own rows
#pragma unroll 1
            for (int rl = lane; rl < R; rl += 32) {
                const int row = r0 + rl;
                const double b = S.b0[rl];
                if (row == n && p.abft) {
                    V[row + (int64_t)j * ldw] = vchk;
                    if (CACHE) Vl[rl * XR + j * XC] = vchk;
                    Apan[row + (int64_t)c * ldw] = (tau != 0.0) ? b - vchk * (alpha - beta) : b;  // left term (R7)
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
                    Apan[row + (int64_t)c * ldw] = av;
                } else if (CACHE) {
                    Vl[rl * XR + j * XC] = 0.0;  // rows outside the panel take no part in the dots
                }
            }
            if (bid == 0 && lane == 0) {
                p.tau[c] = tau;
                if (p.abft) {
                    p.Qc[c] = vchk - 1.0;  // Q column checksum
                    qc_corner += vchk - 1.0;
                }
            }
            // recycle the accumulator set of column c+2 (= that of column c-2): every CTA has
            // finished reading it, and column c+2 adds into it only after two more syncs
            if (bid == 0)
                for (int i = lane; i < FT_ACC_STRIDE; i += 32) p.acc[((c + 2) & 3) * FT_ACC_SET_DOUBLES + i * FT_ACC_PAD] = 0.0;
            PROBE(6);
        }
        {
            // ======================= GEMV, all 16 warps: y = A(:, c+1:) v on the unscaled b ===
            // (warp 0 joins after its DLARFG / V(:, j) work above: with 512 lanes a CTA of 112 rows
            // streams 9 columns at a time instead of 8 -- the CTAs with the most rows set the
            // column's barrier)
            const int gt = tid;
            const int rp = gt % R2p, cl = gt / R2p;
            const bool gemv_on = rp < R2 && cl < ncl;
            const double2 *__restrict__ A2 = reinterpret_cast<const double2 *>(A + r0);
            const int64_t ldw2 = ldw >> 1;
            const double *bv = p.bvec;  // b(q) for c+2 <= q < ihi; zero for q >= ihi
            const bool vfy = (j == 0) && p.verify;
            const int cend = vfy ? n : ihi;
            double2 ya = make_double2(0.0, 0.0), rs = make_double2(0.0, 0.0);
            if (MG && gemv_on && !(p.dbg_mode & 2)) {
                // virtual columns: [0, nA) the panel columns c+2.. (owner only, from Apan), then
                // the local trailing columns lcol0.. (global index J(l) selects x)
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
                // b is read with plain (L1-allocating) loads: the acquire at the grid barrier
                // invalidated this SM's L1 before the trailing bar.sync released us
                int col = c + 2 + cl;
#pragma unroll 1
                for (; col + (GB - 1) * ncl < cend; col += GB * ncl) {
                    double2 a[GB];
                    double v[GB];
#pragma unroll
                    for (int u = 0; u < GB; u++) {
                        const int q = col + u * ncl;
                        a[u] = GLOAD(A2 + (int64_t)q * ldw2 + rp);
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

                if (col < cend) {  // ragged tail: one predicated batch (all loads in flight together)
                    double2 a[GB];
                    double v[GB];
#pragma unroll
                    for (int u = 0; u < GB; u++) {
                        const int q = col + u * ncl;
                        a[u] = q < cend ? GLOAD(A2 + (int64_t)q * ldw2 + rp) : make_double2(0.0, 0.0);
                        v[u] = q < cend ? bv[q] : 0.0;
                    }
#pragma unroll
                    for (int u = 0; u < GB; u++) {
                        ya.x += a[u].x * v[u];
                        ya.y += a[u].y * v[u];
                        rs.x += a[u].x;
                        rs.y += a[u].y;
                    }
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
                    S.red[wid * R2p + lane] = ya;
                    if (vfy) S.rsr[wid * R2p + lane] = rs;
                }
            } else if (cl < ncl) {
                S.red[cl * R2p + rp] = ya;
                if (vfy) S.rsr[cl * R2p + rp] = rs;
            }
        }
        __syncthreads();  // GEMV partials, tau / scale / t, V(:, j) are in shared memory
        if (p.dbg && tid == 0 && j == 8) {  // per-CTA GEMV span (debug hook): smid, start, end, rows
            unsigned long long t1;
            unsigned smid;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
            asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
            p.dbg[2048 + bid * 4 + 0] = smid;
            p.dbg[2048 + bid * 4 + 1] = gt_start;
            p.dbg[2048 + bid * 4 + 2] = t1;
            p.dbg[2048 + bid * 4 + 3] = (unsigned long long)R;
        }
        if (MG) {
            // ---- cross-rank exchange of the GEMV partials, CTA by CTA: every rank
            // uses the same row partition, so CTA bid of each rank owns the same rows.  Push
            // (y partial, A(:, c+1) part) of the own rows into every rank's slot, raise the flag,
            // wait for every rank's flag; phase (v) sums the slots in rank order (identical on
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
                    const double2 u = S.red[q * R2p + pr];
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
            if (wid == 0 && lane < p.G)
                while (ld_acquire_sys_u32(p.flags + lane * FT_FLAG_STRIDE + bid) < seq) {
                }
            __syncthreads();
        }
        PROBE(7);
        // ---------------- (v) Y(:, j) = tau (y - Y t) (an 8-lane group per row) -----------------
        {
            const double tau = S.scal[0], scale = S.scal[2];
            const bool vfy = (j == 0) && p.verify;
            // small row blocks: the T column (warps 8..15) runs beside the Y rows (warps 0..7)
            const bool split = R <= 32;
            if (!split || wid >= 8) {
                // T(a, j) = -tau * sum_{b=a}^{j-1} T(a, b) t(b), T(j, j) = tau (8 lanes per a)
                const int tslot = split ? slot - 32 : slot, tw = split ? wid - 8 : wid;
                const int nsl = split ? 32 : NSLOT;
#pragma unroll 1
                for (int a0 = 0; a0 < j; a0 += nsl) {
                    if (a0 + 4 * tw >= j) break;  // warp-uniform
                    const int a = a0 + tslot;
                    double s0 = 0.0, s1 = 0.0;
                    if (a < j)
#pragma unroll
                        for (int u = 0; u < FT_NBMAX / 8; u += 2) {
                            const int ba = a + g + 8 * u, bb = ba + 8;
                            if (ba < j) s0 += S.Ts[a][ba] * S.t[ba];
                            if (bb < j) s1 += S.Ts[a][bb] * S.t[bb];
                        }
                    const double sT = group8_sum(s0 + s1);
                    if (a < j && g == 0) S.Ts[a][j] = -tau * sT;
                }
            }
            if (tid == 0) S.Ts[j][j] = tau;
            PROBE(12);
            const int rslots = split ? 32 : NSLOT;
#pragma unroll 1
            for (int base = 0; base < R; base += rslots) {
                if (split && wid >= 8) break;
                if (base + 4 * wid >= R) break;
                const int rl = base + slot;
                const bool on = rl < R && is_valid(r0 + rl);
                const int pr = rl >> 1, hi = rl & 1;
                // lane partial of scale * y - Y(rl, :) t: GEMV partials q = g, g + 8 (npart <= 15)
                double ya = 0.0, yb = 0.0, rsum = 0.0, an_mg = 0.0;
                if (on && MG) {
                    if (g == 0) {  // exchanged partials, summed in rank order
                        double ysum = 0.0;
                        const double2 *yxs = p.yx + (int64_t)(c & 1) * p.G * ldw + (r0 + rl);
                        for (int gg = 0; gg < p.G; gg++) {
                            const double2 u = __ldcg(yxs + (int64_t)gg * ldw);
                            ysum += u.x;
                            an_mg += u.y;
                        }
                        ya = scale * ysum;
                    }
                } else if (on) {
#pragma unroll
                    for (int u = 0; u < 2; u++) {
                        const int q = g + 8 * u;
                        if (q < npart) {
                            const double2 w2 = S.red[q * R2p + pr];
                            ya += scale * (hi ? w2.y : w2.x);
                            if (vfy) {
                                const double2 r2 = S.rsr[q * R2p + pr];
                                rsum += hi ? r2.y : r2.x;
                            }
                        }
                    }
                }
                // with the same Y row loads: P1 = Y(rl, :) V(c+1, :)^T (S.vrow), which gives the
                // next column's b0 = A(:, c+1) - Y(:, 0:j) V(c+1, 0:j)^T = an - P1 - Y(:, j)
                double pa = 0.0, pb = 0.0;
                if (on) {
#pragma unroll
                    for (int u = 0; u < FT_NBMAX / 8; u += 2) {
                        const int ja = g + 8 * u, jb = ja + 8;
                        if (ja < j) {
                            const double yv = Yl[rl * XR + ja * XC];
                            ya -= yv * S.t[ja];
                            pa += yv * S.vrow[ja];
                        }
                        if (jb < j) {
                            const double yv = Yl[rl * XR + jb * XC];
                            yb -= yv * S.t[jb];
                            pb += yv * S.vrow[jb];
                        }
                    }
                }
                const double ysum = group8_sum(ya + yb);
                const double p1 = group8_sum(pa + pb);
                if (vfy) rsum = group8_sum(rsum);
                if (rl < R && g == 0) {
                    const int row = r0 + rl;
                    const double an = (MG && c + 1 >= p.e) ? an_mg : S.anext[rl];
                    double b0n = 0.0;
                    if (on) {
                        const double yy = tau * (an + ysum);
                        Y[row + (int64_t)j * ldw] = yy;
                        if (CACHE) Yl[rl * XR + j * XC] = yy;
                        b0n = an - p1 - yy;
                        if (vfy && is_data(row)) {
                            // D_r(row) = r(row) - sum_{col >= k} L(row, col); columns < k are logical zero
                            rsum += S.acol[rl] + an;
                            const double d = p.rcol[row] - rsum;
                            if (not_within(d, tau_abs)) {
                                atomicAdd(&p.ctl->nflag, 1);
                            } else if (tau_abs > 0.0) {
                                const double rel = fabs(d) / (tau_abs / c_thr);
                                atomicMax(&S.drift, (unsigned long long)__double_as_longlong(rel));  // smem: one global max per CTA
                            }
                        }
                    }
                    S.acol[rl] = an;
                    S.b0[rl] = b0n;
                    S.bm[rl] = is_data(row) ? b0n : 0.0;
                }
            }
            PROBE(13);
            __syncthreads();
        }
        PROBE(8);
    }
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
    if (p.precheck_sums) {  // e^T Y, e^T V over the own data rows (pre-update check R15, fused): 4 lanes per sum
        const int o = tid >> 2, q = tid & 3, jj = o % ib;
        const double *X = o < ib ? Yl : Vl;
        double s = 0.0;
        if (o < 2 * ib)
            for (int rl = q; rl < R; rl += 4)
                if (is_data(r0 + rl)) s += X[rl * XR + jj * XC];
        s += __shfl_xor_sync(0xffffffffu, s, 1);
        s += __shfl_xor_sync(0xffffffffu, s, 2);
        if (q == 0 && o < 2 * ib) atomicAdd(o < ib ? &p.ctl->eY[jj * FT_ESTR] : &p.ctl->eV[jj * FT_ESTR], s);
    }
    if (bid == 0 && tid == 0 && p.abft) atomicAdd(&p.Qc[n], qc_corner);  // single writer: Qc(n) + corner
    // T, max |T| and the T checksum from three different CTAs (every CTA holds T in shared memory)
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
}

cudaError_t ft_launch_panel_wide(const PanelLaunch &L, int nsm, cudaStream_t s) {
    static int max_smem = 0;
    static unsigned attr = 0;
    const unsigned dbit = ft_dev_bit();
    if (!(attr & dbit)) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&max_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        const void *fns[] = {(const void *)k_panel_wide<true, false>, (const void *)k_panel_wide<false, false>};
        for (const void *fn : fns) {
            cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, max_smem);
            if (e != cudaSuccess) return e;
        }
        attr |= dbit;
    }
    if (L.nr != 1) return cudaErrorInvalidValue;
    PanelLaunch Lw = L;  // ngroups in GR-row units (rbase is a multiple of GR_DRIVER)
    Lw.r[0].ngroups = L.r[0].ngroups * (GR_DRIVER / GR);
    int grid = nsm < L.r[0].ngroups ? nsm : L.r[0].ngroups;
    if (grid > FT_FLAG_STRIDE) grid = FT_FLAG_STRIDE;
    if (grid < 1) grid = 1;
    const int gmax = (Lw.r[0].ngroups + grid - 1) / grid;
    const int rmax = GR * gmax;
    if (rmax > RMAX) return cudaErrorInvalidConfiguration;
    const size_t fixed = sizeof(PanelSmemW);
    const size_t want = fixed + (size_t)2 * VS * rmax * sizeof(double);
    const bool cache = want <= (size_t)max_smem;
    if (L.r[0].dpart && grid > FT_DPMAX) return cudaErrorInvalidValue;  // deterministic mode: partial slots
    void *args[] = {&Lw};
    g_ft_launches++;
    g_ft_wide_launches++;
    const void *fn = cache ? (const void *)k_panel_wide<true, false> : (const void *)k_panel_wide<false, false>;
    return cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(PT), args, cache ? want : fixed, s);
}
