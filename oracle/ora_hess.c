/*
 * ora_hess.c -- the CPU oracle (TEST INFRASTRUCTURE ONLY; see oracle.h).
 *
 * What each function follows:
 *   ora_dgehd2    unblocked Householder reduction H = Q^T A Q          P:38-40 (Sec. III-A)
 *                 with LAPACK DLARFG/DGEHD2 conventions (reading R1, R3)
 *   ora_dorghr    Q = H(ilo) ... H(ihi-1), backward accumulation         P:40 (Q = Q1 Q2 ... Qn)
 *   encode        r = A e, c = e^T A, kappa = e^T A e                    P:218-224 (Sec. IV-B, Fig. 3), R22
 *   bookkeeping   Theorem 1 applied per reflector (right then left)      P:268-274 (Sec. IV-D)
 *   verify        recompute L e, e^T L at each boundary                  P:256-260, P:272 (Sec. IV-C/F)
 *   decode/fix    A(i,j) = r(i) - sum_{k!=j} A(i,k) (or column form)     P:278 (Sec. IV-F), R12
 *   Q protection  Qr/Qc of the Householder vectors, checked at the end   P:266, P:278 (Sec. IV-E)
 *   injector      XOR one bit of a binary64 word                         P:48-52 (failure model), R16
 *
 * The paper checks once per nb-column iteration (Alg. 3 l.12-13);
 * the oracle runs the unblocked algorithm and verifies at the same
 * boundaries (columns k = ilo-1 + t*nb) with the vector test of R11,
 * recomputing the checksums from scratch (no fusion, no incremental sums).
 */
#include "oracle.h"

#include <float.h>
#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define AT(A, lda, i, j) (A)[(size_t)(i) + (size_t)(j) * (size_t)(lda)]
/* rows per block of the streamed row-wise sums (memory order only): one block per thread,
 * a multiple of 8 rows, at most 4096 (the block's accumulators stay in L2) */
static int row_block(int m) {
    int nt = 1;
#ifdef _OPENMP
    nt = omp_get_max_threads();
#endif
    int rb = (m + nt - 1) / nt;
    rb = (rb + 7) / 8 * 8;
    if (rb > 4096) rb = 4096;
    return rb < 8 ? 8 : rb;
}
static const double EPS = DBL_EPSILON; /* 2^-52, R17 */

int ora_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

double ora_flip(double *x, int bit) {
    uint64_t u;
    double old = *x;
    memcpy(&u, x, 8);
    u ^= (uint64_t)1 << (bit & 63);
    memcpy(x, &u, 8);
    return *x - old;
}

/* ------------------------------------------------------------------ */
/* DLARFG (R1): given alpha and x (length m), produce beta, tau and     */
/* scale x in place so that H [alpha; x] = [beta; 0], H = I - tau v v^T, */
/* v = [1; x_scaled].  xnorm = 0 (or m = 0) gives tau = 0, H = I.        */
/* ------------------------------------------------------------------ */
static void dlarfg(int m, double *alpha, double *x, double *tau) {
    double xnorm2 = 0.0;
    for (int i = 0; i < m; i++) xnorm2 += x[i] * x[i];
    double xnorm = sqrt(xnorm2);
    if (m <= 0 || xnorm == 0.0) {
        *tau = 0.0;
        return;
    }
    double beta = -copysign(hypot(*alpha, xnorm), *alpha);
    *tau = (beta - *alpha) / beta;
    double scal = 1.0 / (*alpha - beta);
    for (int i = 0; i < m; i++) x[i] *= scal;
    *alpha = beta;
}

static int check_args(int n, int ilo, int ihi, const void *A, int lda, const void *tau) {
    if (n < 0) return -1;
    if (ilo < 1 || ilo > (n > 1 ? n : 1)) return -2;
    if (ihi < (ilo < n ? ilo : n) || ihi > n) return -3;
    if (n > 0 && A == NULL) return -4;
    if (lda < (n > 1 ? n : 1)) return -5;
    if (n > 1 && tau == NULL) return -6;
    return 0;
}

/* One reflector step at column c (0-based), optionally carrying the
 * checksum bookkeeping of Theorem 1.  y, w are workspaces of length n.
 * Returns tau.  chk == NULL: plain DGEHD2 step. */
typedef struct {
    double *r, *c, *kap;     /* H checksums (length n, n, 1) */
    double *qr, *qc, *qk;    /* Q checksums */
    /* weighted pair (NEXT-1), w_i = i + 1, or NULL: r_w = L w, c_w = w^T L and the corners
     * krw = e^T L w, kcw = w^T L e */
    double *rw, *cw, *krw, *kcw;
} chk_t;

#define WGT(i) ((double)(i) + 1.0) /* weight of 0-based index i (NEXT-1) */

static double reflector_step(int n, int ihi, double *A, int lda, int c,
                             double *y, double *w, chk_t *chk) {
    int m = ihi - c - 1;                 /* length of [alpha; x] = rows c+1..ihi-1 */
    double tau = 0.0;
    if (m < 1) return 0.0;
    double *alpha = &AT(A, lda, c + 1, c);
    double *x = &AT(A, lda, c + 2, c);   /* rows c+2..ihi-1, length m-1 */
    double alpha0 = *alpha;
    dlarfg(m - 1, alpha, x, &tau);
    if (tau == 0.0) {
        if (chk) {                       /* H(c) = I: checksums unchanged, Qc(c) = sum x */
            double sx = 0.0;
            for (int i = 0; i < m - 1; i++) sx += x[i];
            chk->qc[c] = sx;
            for (int i = 0; i < m - 1; i++) chk->qr[c + 2 + i] += x[i];
            *chk->qk += sx;
        }
        return 0.0;
    }
    double beta = *alpha;
    /* v(c+1) = 1 implicit, v(c+2:ihi) = x */
#define V(i) ((i) == c + 1 ? 1.0 : AT(A, lda, (i), c))
    double ev = 1.0;                     /* e^T v */
    for (int i = c + 2; i < ihi; i++) ev += V(i);

    double wv = WGT(c + 1);              /* w^T v (weighted pair) */
    for (int i = c + 2; i < ihi; i++) wv += WGT(i) * V(i);
    if (chk) {
        /* reduced column c: left term of its own reflector (R7): c[c] -= (e^T v)(alpha - beta) */
        chk->c[c] -= ev * (alpha0 - beta);
        if (chk->rw) chk->cw[c] -= wv * (alpha0 - beta);
        /* Q checksums of the new Householder vector (Fig. 5) */
        chk->qc[c] = ev - 1.0;
        for (int i = c + 2; i < ihi; i++) chk->qr[i] += V(i);
        *chk->qk += ev - 1.0;
    }

    /* Right step: A(0:ihi, c+1:ihi) := A (I - tau v v^T).  y = A v.  P:38 (A Q_i)
     * y(i) = sum_j A(i,j) v(j), j increasing -- the loop nest runs j-outer over a block of
     * rows so the column-major matrix streams; every y(i) sees the same additions in the
     * same order as the plain dot (bitwise identical; -ffp-contract=off). */
#pragma omp parallel for schedule(static)
    for (int i0 = 0; i0 < ihi; i0 += row_block(ihi)) {
        const int rb = row_block(ihi), i1 = i0 + rb < ihi ? i0 + rb : ihi;
        for (int i = i0; i < i1; i++) y[i] = 0.0;
        for (int j = c + 1; j < ihi; j++) {
            const double vj = V(j);
            for (int i = i0; i < i1; i++) y[i] += AT(A, lda, i, j) * vj;
        }
    }
    if (chk) {
        /* Theorem 1 part 2 at reflector granularity */
        double cv = 0.0;
        for (int j = c + 1; j < ihi; j++) cv += chk->c[j] * V(j);
        *chk->kap -= tau * cv * ev;
        if (chk->rw) {
            /* the same algebra with w: r_w' = A (I - tau v v^T) w = r_w - tau (w^T v) y,
             * c_w' = c_w - tau (c_w.v) v^T, e^T A' w and w^T A' e likewise */
            double cwv = 0.0;
            for (int j = c + 1; j < ihi; j++) cwv += chk->cw[j] * V(j);
            *chk->krw -= tau * cv * wv;
            *chk->kcw -= tau * cwv * ev;
            for (int j = c + 1; j < ihi; j++) chk->cw[j] -= tau * cwv * V(j);
            for (int i = 0; i < ihi; i++) chk->rw[i] -= tau * wv * y[i];
        }
        for (int j = c + 1; j < ihi; j++) chk->c[j] -= tau * cv * V(j);
        for (int i = 0; i < ihi; i++) chk->r[i] -= tau * ev * y[i];
    }
#pragma omp parallel for schedule(static)
    for (int j = c + 1; j < ihi; j++) {
        double vj = tau * V(j);
        for (int i = 0; i < ihi; i++) AT(A, lda, i, j) -= y[i] * vj;
    }

    /* Left step: A(c+1:ihi, c+1:n) := (I - tau v v^T) A.  w = v^T A.  P:38 (Q_i^{-1} A) */
#pragma omp parallel for schedule(static)
    for (int j = c + 1; j < n; j++) {
        double s = 0.0;
        for (int i = c + 1; i < ihi; i++) s += V(i) * AT(A, lda, i, j);
        w[j] = s;
    }
    if (chk) {
        /* Theorem 1 part 3 at reflector granularity */
        double vr = 0.0;
        for (int i = c + 1; i < ihi; i++) vr += V(i) * chk->r[i];
        *chk->kap -= tau * ev * vr;
        if (chk->rw) {
            /* r_w' = (I - tau v v^T) r_w, c_w' = c_w - tau (w^T v) (v^T A), corners likewise */
            double vrw = 0.0;
            for (int i = c + 1; i < ihi; i++) vrw += V(i) * chk->rw[i];
            *chk->krw -= tau * ev * vrw;
            *chk->kcw -= tau * wv * vr;
            for (int i = c + 1; i < ihi; i++) chk->rw[i] -= tau * vrw * V(i);
            for (int j = c + 1; j < n; j++) chk->cw[j] -= tau * wv * w[j];
        }
        for (int i = c + 1; i < ihi; i++) chk->r[i] -= tau * vr * V(i);
        for (int j = c + 1; j < n; j++) chk->c[j] -= tau * ev * w[j];
    }
#pragma omp parallel for schedule(static)
    for (int j = c + 1; j < n; j++) {
        double wj = tau * w[j];
        for (int i = c + 1; i < ihi; i++) AT(A, lda, i, j) -= V(i) * wj;
    }
#undef V
    return tau;
}

int ora_dgehd2(int n, int ilo, int ihi, double *A, int lda, double *tau) {
    int info = check_args(n, ilo, ihi, A, lda, tau);
    if (info) return info;
    for (int c = 0; c < n - 1; c++) tau[c] = 0.0;
    if (n <= 1) return 0;
    double *y = (double *)calloc((size_t)n, sizeof(double));
    double *w = (double *)calloc((size_t)n, sizeof(double));
    for (int c = ilo - 1; c <= ihi - 2; c++) tau[c] = reflector_step(n, ihi, A, lda, c, y, w, NULL);
    free(y);
    free(w);
    return 0;
}

int ora_dorghr(int n, int ilo, int ihi, const double *A, int lda, const double *tau,
               double *Q, int ldq) {
    int info = check_args(n, ilo, ihi, A, lda, tau);
    if (info) return info;
    if (Q == NULL) return -7;
    if (ldq < (n > 1 ? n : 1)) return -8;
    for (int j = 0; j < n; j++)
        for (int i = 0; i < n; i++) AT(Q, ldq, i, j) = (i == j) ? 1.0 : 0.0;
    if (n <= 1) return 0;
    double *w = (double *)calloc((size_t)n, sizeof(double));
    /* Q := H(c) Q for c = ihi-2 down to ilo-1; H(c) acts on rows/cols c+1..ihi-1 */
    for (int c = ihi - 2; c >= ilo - 1; c--) {
        double t = tau[c];
        if (t == 0.0) continue;
#define V(i) ((i) == c + 1 ? 1.0 : AT(A, lda, (i), c))
#pragma omp parallel for schedule(static)
        for (int j = c + 1; j < ihi; j++) {
            double s = 0.0;
            for (int i = c + 1; i < ihi; i++) s += V(i) * AT(Q, ldq, i, j);
            w[j] = s;
        }
#pragma omp parallel for schedule(static)
        for (int j = c + 1; j < ihi; j++) {
            double wj = t * w[j];
            for (int i = c + 1; i < ihi; i++) AT(Q, ldq, i, j) -= V(i) * wj;
        }
#undef V
    }
    free(w);
    return 0;
}

/* ------------------------------------------------------------------ */
/* Decoder (reading R12, "decoder v2"): never miscorrect.              */
/* ------------------------------------------------------------------ */
static void push_ev(ora_report *rep, int kind, int panel, int64_t i, int64_t j, double delta) {
    if (!rep) return;
    if (rep->nevents < ORA_MAX_EVENTS) {
        ora_event *e = &rep->ev[rep->nevents++];
        e->kind = kind; e->panel = panel; e->i = i; e->j = j; e->delta = delta;
    }
}

static int bad(double d, double tau) { return !(fabs(d) <= tau); } /* NaN counts as flagged */

static int approx(double a, double b, double tol) {
    if (!isfinite(a) || !isfinite(b)) return !isfinite(a) && !isfinite(b);
    return fabs(a - b) <= tol;
}

typedef struct { double *Dr, *Dc, sr, sc; } syn_t;

/* row sums t(i) = sum_j L(i,j), j increasing (blocked over rows, column-major streaming;
 * the same order of additions as the plain per-row loop) */
static void row_sums(int n, const double *L, int ldl, double *t) {
#pragma omp parallel for schedule(static)
    for (int i0 = 0; i0 < n; i0 += row_block(n)) {
        const int rb = row_block(n), i1 = i0 + rb < n ? i0 + rb : n;
        for (int i = i0; i < i1; i++) t[i] = 0.0;
        for (int j = 0; j < n; j++)
            for (int i = i0; i < i1; i++) t[i] += AT(L, ldl, i, j);
    }
}

static void syndromes(int n, const double *L, int ldl, const double *r, const double *c,
                      double kap, syn_t *s) {
    row_sums(n, L, ldl, s->Dr);
    for (int i = 0; i < n; i++) s->Dr[i] = r[i] - s->Dr[i];
#pragma omp parallel for schedule(static)
    for (int j = 0; j < n; j++) {
        double t = 0.0;
        for (int i = 0; i < n; i++) t += AT(L, ldl, i, j);
        s->Dc[j] = c[j] - t;
    }
    double sr = 0.0, sc = 0.0;
    for (int i = 0; i < n; i++) sr += r[i];
    for (int j = 0; j < n; j++) sc += c[j];
    s->sr = sr - kap;
    s->sc = sc - kap;
}

/* unique subset S' of idx[0..m) (size <= 3) with sum D over S' ~ target.
 * Returns size (0..3) with members in out[], or -1 if none / not unique. */
static int unique_subset(int m, const int *idx, const double *D, double target,
                         double tauS, int n, int *out) {
    double tol_base = tauS;
    if (approx(target, 0.0, tauS)) return 0;
    if (!isfinite(target)) {       /* a checksum word became inf/nan: take the non-finite ones */
        int k = 0;
        for (int a = 0; a < m; a++)
            if (!isfinite(D[idx[a]])) { if (k == 3) return -1; out[k++] = idx[a]; }
        return k > 0 ? k : -1;
    }
    if (m > 256) return -1;
    int found = 0, best[3] = {-1, -1, -1}, bsz = 0;
    for (int a = 0; a < m; a++) {
        double da = D[idx[a]];
        double tol = tol_base + 2.0 * n * EPS * fabs(da);
        if (approx(da, target, tol)) { found++; best[0] = idx[a]; bsz = 1; }
        for (int b = a + 1; b < m; b++) {
            double db = D[idx[b]];
            double tol2 = tol_base + 2.0 * n * EPS * (fabs(da) + fabs(db));
            if (approx(da + db, target, tol2)) { found++; best[0] = idx[a]; best[1] = idx[b]; bsz = 2; }
            for (int e = b + 1; e < m; e++) {
                double de = D[idx[e]];
                double tol3 = tol_base + 2.0 * n * EPS * (fabs(da) + fabs(db) + fabs(de));
                if (approx(da + db + de, target, tol3)) {
                    found++; best[0] = idx[a]; best[1] = idx[b]; best[2] = idx[e]; bsz = 3;
                }
            }
        }
    }
    if (found != 1) return -1;
    for (int k = 0; k < bsz; k++) out[k] = best[k];
    return bsz;
}

static int in_set(int v, const int *s, int m) {
    for (int k = 0; k < m; k++) if (s[k] == v) return 1;
    return 0;
}

/* A(i,j) = r(i) - sum_{k != j} L(i,k)   (first formula) */
static double fix_row(int n, double *L, int ldl, const double *r, int i, int j) {
    double s = 0.0;
    for (int k = 0; k < n; k++) if (k != j) s += AT(L, ldl, i, k);
    double old = AT(L, ldl, i, j);
    AT(L, ldl, i, j) = r[i] - s;
    return AT(L, ldl, i, j) - old;
}
/* A(i,j) = c(j) - sum_{k != i} L(k,j)   (second formula) */
static double fix_col(int n, double *L, int ldl, const double *c, int i, int j) {
    double s = 0.0;
    for (int k = 0; k < n; k++) if (k != i) s += AT(L, ldl, k, j);
    double old = AT(L, ldl, i, j);
    AT(L, ldl, i, j) = c[j] - s;
    return AT(L, ldl, i, j) - old;
}

int ora_decode(int n, double *L, int ldl, double *r, double *c, double *kappa,
               double tau_abs, ora_report *rep, int panel, int mode) {
    const int evD = mode == ORA_MODE_Q ? ORA_EV_FIX_Q : ORA_EV_FIX_DATA;
    const int evR = mode == ORA_MODE_Q ? ORA_EV_FIX_QR : ORA_EV_FIX_R;
    const int evC = mode == ORA_MODE_Q ? ORA_EV_FIX_QC : ORA_EV_FIX_C;
    const int evK = mode == ORA_MODE_Q ? ORA_EV_FIX_QK : ORA_EV_FIX_K;
    double tauS = tau_abs * sqrt((double)(n > 1 ? n : 1));
    syn_t s;
    s.Dr = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
    s.Dc = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
    int *R = (int *)malloc(sizeof(int) * (size_t)(n > 0 ? n : 1));
    int *C = (int *)malloc(sizeof(int) * (size_t)(n > 0 ? n : 1));
    int *Rd = (int *)malloc(sizeof(int) * (size_t)(n > 0 ? n : 1));
    int *Cd = (int *)malloc(sizeof(int) * (size_t)(n > 0 ? n : 1));
    int result = 0;
    syndromes(n, L, ldl, r, c, *kappa, &s);
    int nR = 0, nC = 0;
    for (int i = 0; i < n; i++) if (bad(s.Dr[i], tau_abs)) R[nR++] = i;
    for (int j = 0; j < n; j++) if (bad(s.Dc[j], tau_abs)) C[nC++] = j;
    int sr_ok = approx(s.sr, 0.0, tauS), sc_ok = approx(s.sc, 0.0, tauS);
    if (nR == 0 && nC == 0 && sr_ok && sc_ok) { result = 0; goto done; }
    push_ev(rep, ORA_EV_DETECT, panel, nR, nC, 0.0);
    if (rep) rep->detected++;

    if (nR == 0 && nC == 0) {
        /* (1) only the corner disagrees: both sums off by the same amount */
        if (!sr_ok && !sc_ok && approx(s.sr, s.sc, tauS)) {
            double sr = 0.0;
            for (int i = 0; i < n; i++) sr += r[i];
            double old = *kappa;
            *kappa = sr;
            push_ev(rep, evK, panel, -1, -1, *kappa - old);
        } else {
            result = 2;
            goto done;
        }
    } else {
        /* (2) checksum-vector errors: unique subset whose syndrome sum explains s_r / s_c.
         * If s_r ~ s_c != 0 the same syndrome is also produced by a corner error
         * plus data errors (e.g. r(i), c(j) both off by -d  ==  A(i,j) and kappa
         * both off by +d): information-theoretically ambiguous, so refuse. */
        if (!sr_ok && !sc_ok && approx(s.sr, s.sc, tauS)) { result = 2; goto done; }
        int Rc[3], Cc[3];
        int nRc = unique_subset(nR, R, s.Dr, s.sr, tauS, n, Rc);
        int nCc = unique_subset(nC, C, s.Dc, s.sc, tauS, n, Cc);
        if (nRc < 0 || nCc < 0) { result = 2; goto done; }
        int nRd = 0, nCd = 0;
        for (int a = 0; a < nR; a++) if (!in_set(R[a], Rc, nRc)) Rd[nRd++] = R[a];
        for (int a = 0; a < nC; a++) if (!in_set(C[a], Cc, nCc)) Cd[nCd++] = C[a];
        /* A flagged line with no flagged partner can only be a checksum word: when its
         * syndrome hid inside the sum tolerance (tau < |d| <= tau*sqrt(n)), take the whole
         * flagged set as checksum errors if it explains s_r (s_c) within that tolerance. */
        if (nRd > 0 && nCd == 0 && nR <= 3) {
            double sum = 0.0, sa = 0.0;
            int small = 1; /* only syndromes that could hide inside tauS (not a cancelling pair) */
            for (int a = 0; a < nR; a++) { sum += s.Dr[R[a]]; sa += fabs(s.Dr[R[a]]); small &= fabs(s.Dr[R[a]]) <= tauS; }
            if (small && approx(sum, s.sr, tauS + 2.0 * n * EPS * sa)) {
                nRc = nR;
                for (int a = 0; a < nR; a++) Rc[a] = R[a];
                nRd = 0;
            }
        }
        if (nCd > 0 && nRd == 0 && nC <= 3) {
            double sum = 0.0, sa = 0.0;
            int small = 1;
            for (int a = 0; a < nC; a++) { sum += s.Dc[C[a]]; sa += fabs(s.Dc[C[a]]); small &= fabs(s.Dc[C[a]]) <= tauS; }
            if (small && approx(sum, s.sc, tauS + 2.0 * n * EPS * sa)) {
                nCc = nC;
                for (int a = 0; a < nC; a++) Cc[a] = C[a];
                nCd = 0;
            }
        }
        /* (3) data errors */
        if (nRd == 0 && nCd == 0) {
            /* only checksum words were hit */
        } else if (nRd == 0 || nCd == 0) {
            result = 2; goto done;
        } else if (nRd == 1 && nCd == 1) {
            double tol = 2.0 * tau_abs + 2.0 * n * EPS * (fabs(s.Dr[Rd[0]]) + fabs(s.Dc[Cd[0]]));
            if (!approx(s.Dr[Rd[0]], s.Dc[Cd[0]], tol)) { result = 2; goto done; }
            double d = fix_row(n, L, ldl, r, Rd[0], Cd[0]);
            push_ev(rep, evD, panel, Rd[0], Cd[0], d);
        } else if (nRd == 1) {
            /* one shared row, several columns: column formulas */
            double sum = 0.0, sabs = 0.0;
            int nonfin = 0;
            for (int b = 0; b < nCd; b++) { sum += s.Dc[Cd[b]]; sabs += fabs(s.Dc[Cd[b]]); nonfin |= !isfinite(s.Dc[Cd[b]]); }
            double tol = 2.0 * tauS + 2.0 * n * EPS * (sabs + fabs(s.Dr[Rd[0]]));
            if (!nonfin && !approx(sum, s.Dr[Rd[0]], tol)) { result = 2; goto done; }
            if (nonfin && isfinite(s.Dr[Rd[0]])) { result = 2; goto done; }
            for (int b = 0; b < nCd; b++) {
                double d = fix_col(n, L, ldl, c, Rd[0], Cd[b]);
                push_ev(rep, evD, panel, Rd[0], Cd[b], d);
            }
        } else if (nCd == 1) {
            /* one shared column, several rows: row formulas */
            double sum = 0.0, sabs = 0.0;
            int nonfin = 0;
            for (int a = 0; a < nRd; a++) { sum += s.Dr[Rd[a]]; sabs += fabs(s.Dr[Rd[a]]); nonfin |= !isfinite(s.Dr[Rd[a]]); }
            double tol = 2.0 * tauS + 2.0 * n * EPS * (sabs + fabs(s.Dc[Cd[0]]));
            if (!nonfin && !approx(sum, s.Dc[Cd[0]], tol)) { result = 2; goto done; }
            if (nonfin && isfinite(s.Dc[Cd[0]])) { result = 2; goto done; }
            for (int a = 0; a < nRd; a++) {
                double d = fix_row(n, L, ldl, r, Rd[a], Cd[0]);
                push_ev(rep, evD, panel, Rd[a], Cd[0], d);
            }
        } else if (nRd == nCd) {
            /* distinct rows and columns: pair by value, uniquely in both directions */
            int *pair = (int *)malloc(sizeof(int) * (size_t)nRd);
            int okp = 1;
            for (int a = 0; a < nRd && okp; a++) {
                int cnt = 0;
                for (int b = 0; b < nCd; b++) {
                    double tol = 2.0 * tau_abs + 2.0 * n * EPS * (fabs(s.Dr[Rd[a]]) + fabs(s.Dc[Cd[b]]));
                    if (approx(s.Dr[Rd[a]], s.Dc[Cd[b]], tol)) { cnt++; pair[a] = b; }
                }
                if (cnt != 1) okp = 0;
            }
            for (int b = 0; b < nCd && okp; b++) {
                int cnt = 0;
                for (int a = 0; a < nRd; a++) {
                    double tol = 2.0 * tau_abs + 2.0 * n * EPS * (fabs(s.Dr[Rd[a]]) + fabs(s.Dc[Cd[b]]));
                    if (approx(s.Dr[Rd[a]], s.Dc[Cd[b]], tol)) cnt++;
                }
                if (cnt != 1) okp = 0;
            }
            if (okp)
                for (int a = 0; a < nRd; a++) {
                    double d = fix_row(n, L, ldl, r, Rd[a], Cd[pair[a]]);
                    push_ev(rep, evD, panel, Rd[a], Cd[pair[a]], d);
                }
            free(pair);
            if (!okp) { result = 2; goto done; }
        } else {
            result = 2; goto done;
        }
        /* (4) refresh the corrupted checksum words from the (repaired) data */
        for (int a = 0; a < nRc; a++) {
            int i = Rc[a];
            double t = 0.0;
            for (int j = 0; j < n; j++) t += AT(L, ldl, i, j);
            double old = r[i];
            r[i] = t;
            push_ev(rep, evR, panel, i, -1, r[i] - old);
        }
        for (int b = 0; b < nCc; b++) {
            int j = Cc[b];
            double t = 0.0;
            for (int i = 0; i < n; i++) t += AT(L, ldl, i, j);
            double old = c[j];
            c[j] = t;
            push_ev(rep, evC, panel, -1, j, c[j] - old);
        }
    }
    /* (5) re-verify: anything left is uncorrectable */
    syndromes(n, L, ldl, r, c, *kappa, &s);
    result = 1;
    for (int i = 0; i < n && result == 1; i++) if (bad(s.Dr[i], tau_abs)) result = 2;
    for (int j = 0; j < n && result == 1; j++) if (bad(s.Dc[j], tau_abs)) result = 2;
    if (result == 1 && !(approx(s.sr, 0.0, tauS) && approx(s.sc, 0.0, tauS))) result = 2;
done:
    if (result == 1 && rep) rep->corrected++;
    if (result == 2) {
        push_ev(rep, ORA_EV_UNCORRECTABLE, panel, nR, nC, 0.0);
        if (rep) rep->uncorrectable++;
    }
    free(s.Dr); free(s.Dc); free(R); free(C); free(Rd); free(Cd);
    return result;
}

/* ------------------------------------------------------------------ */
/* Weighted checksum pair (NEXT-1): w_i = i + 1.           */
/* r_w = L w, c_w = w^T L, krw = e^T L w, kcw = w^T L e.                 */
/* ------------------------------------------------------------------ */
static void encode_w(int n, const double *L, int ldl, double *rw, double *cw, double *krw, double *kcw) {
#pragma omp parallel for schedule(static)
    for (int i0 = 0; i0 < n; i0 += row_block(n)) {
        const int rb = row_block(n), i1 = i0 + rb < n ? i0 + rb : n;
        for (int i = i0; i < i1; i++) rw[i] = 0.0;
        for (int j = 0; j < n; j++) {
            const double wj = WGT(j);
            for (int i = i0; i < i1; i++) rw[i] += AT(L, ldl, i, j) * wj;
        }
    }
#pragma omp parallel for schedule(static)
    for (int j = 0; j < n; j++) {
        double t = 0.0;
        for (int i = 0; i < n; i++) t += WGT(i) * AT(L, ldl, i, j);
        cw[j] = t;
    }
    double a = 0.0, b = 0.0;
    for (int i = 0; i < n; i++) a += rw[i];
    for (int j = 0; j < n; j++) b += cw[j];
    *krw = a;
    *kcw = b;
}

/* weighted row / column sum of one line (explicit, for refreshes) */
static double row_w(int n, const double *L, int ldl, int i) {
    double t = 0.0;
    for (int j = 0; j < n; j++) t += AT(L, ldl, i, j) * WGT(j);
    return t;
}
static double col_w(int n, const double *L, int ldl, int j) {
    double t = 0.0;
    for (int i = 0; i < n; i++) t += WGT(i) * AT(L, ldl, i, j);
    return t;
}
static double row_e(int n, const double *L, int ldl, int i) {
    double t = 0.0;
    for (int j = 0; j < n; j++) t += AT(L, ldl, i, j);
    return t;
}
static double col_e(int n, const double *L, int ldl, int j) {
    double t = 0.0;
    for (int i = 0; i < n; i++) t += AT(L, ldl, i, j);
    return t;
}

/* the index a weighted / plain syndrome ratio names: D_w / D = w_x = x + 1 for a single error at
 * x; -1 unless the ratio is within 1/4 of an integer in [1, n] after its rounding error
 * (|D_w| <= tw, |D| <= t: ratio error <= (tw + n t) / |D|) */
static int ratio_index(double Dw, double D, double t, double tw, int n) {
    if (!isfinite(Dw) || !isfinite(D) || !(fabs(D) > t)) return -1;
    const double rho = Dw / D;
    const double err = (tw + (double)n * t) / fabs(D) + 4.0 * n * EPS * fabs(rho);
    if (!(err < 0.25)) return -1;
    const double k = nearbyint(rho);
    if (!(fabs(rho - k) <= err) || k < 1.0 || k > (double)n) return -1;
    return (int)k - 1;
}

/* Decoder v3 (weighted pair).  First the paper's single pair (v2, R12) on L, r, c, kappa: if it
 * corrects (or finds nothing), only weighted checksum words can still disagree -- they are
 * refreshed from the verified data.  If v2 refuses (value ties, L-shapes), the weighted pair
 * locates: a column j whose syndromes satisfy D_cw(j) / D_c(j) = w_i holds its one error at row i
 * (and a row likewise), which needs no pairing by value.  Every located error is repaired with
 * an explicit sum along the line that holds no other error; checksum words whose line
 * shows no data error are refreshed; everything is re-verified and any remaining discrepancy is
 * reported uncorrectable (never a wrong correction).  Returns 0 clean, 1 corrected, 2 refused. */
int ora_decode_w(int n, double *L, int ldl, double *r, double *c, double *kappa, double *rw, double *cw,
                 double *krw, double *kcw, double tau_abs, ora_report *rep, int panel) {
    const size_t nn = (size_t)(n > 0 ? n : 1);
    const double tw = tau_abs * (double)n;           /* weighted sums: weights up to n */
    const double tauS = tau_abs * sqrt((double)(n > 1 ? n : 1)), twS = tw * sqrt((double)(n > 1 ? n : 1));
    /* keep the input: v2 may modify L before refusing */
    double *L0 = (double *)malloc(sizeof(double) * nn * nn), *r0 = (double *)malloc(sizeof(double) * nn),
           *c0 = (double *)malloc(sizeof(double) * nn);
    for (int j = 0; j < n; j++)
        for (int i = 0; i < n; i++) L0[i + (size_t)j * nn] = AT(L, ldl, i, j);
    memcpy(r0, r, sizeof(double) * nn);
    memcpy(c0, c, sizeof(double) * nn);
    const double k0 = *kappa;
    const int nev0 = rep ? rep->nevents : 0, det0 = rep ? rep->detected : 0, cor0 = rep ? rep->corrected : 0,
              unc0 = rep ? rep->uncorrectable : 0;
    int result = ora_decode(n, L, ldl, r, c, kappa, tau_abs, rep, panel, ORA_MODE_H);
    double *Dr = (double *)malloc(sizeof(double) * nn), *Dc = (double *)malloc(sizeof(double) * nn);
    double *Drw = (double *)malloc(sizeof(double) * nn), *Dcw = (double *)malloc(sizeof(double) * nn);
    int *pi = (int *)malloc(sizeof(int) * nn);
    int detected_here = 0;
    if (result == 2) {
        /* ---- weighted location on the original input ---- */
        for (int j = 0; j < n; j++)
            for (int i = 0; i < n; i++) AT(L, ldl, i, j) = L0[i + (size_t)j * nn];
        memcpy(r, r0, sizeof(double) * nn);
        memcpy(c, c0, sizeof(double) * nn);
        *kappa = k0;
        if (rep) { /* the single-pair attempt's events are replaced by this decode's */
            rep->nevents = nev0; rep->detected = det0; rep->corrected = cor0; rep->uncorrectable = unc0;
        }
        result = 1;
        for (int pass = 0; pass < 8; pass++) {  /* each pass can free lines for the next (L-shapes) */
        for (int i = 0; i < n; i++) { Dr[i] = r[i] - row_e(n, L, ldl, i); Drw[i] = rw[i] - row_w(n, L, ldl, i); }
        for (int j = 0; j < n; j++) { Dc[j] = c[j] - col_e(n, L, ldl, j); Dcw[j] = cw[j] - col_w(n, L, ldl, j); }
        int nR = 0, nC = 0;
        for (int i = 0; i < n; i++) nR += bad(Dr[i], tau_abs);
        for (int j = 0; j < n; j++) nC += bad(Dc[j], tau_abs);
        if (pass == 0) {
            push_ev(rep, ORA_EV_DETECT, panel, nR, nC, 0.0);
            if (rep) rep->detected++;
            detected_here = 1;
        }
        if (nR == 0 || nC == 0) break;
        /* candidates: column j names row pi[j]; row i names column ratio_index(...).  A named
         * line must itself be flagged (plain or weighted syndrome: a pair cancelling in the plain
         * sum of a line never cancels in its weighted sum, w_j1 != w_j2) */
        for (int j = 0; j < n; j++) {
            pi[j] = -1;
            if (!bad(Dc[j], tau_abs)) continue;
            const int i = ratio_index(Dcw[j], Dc[j], tau_abs, tw, n);
            if (i >= 0 && (bad(Dr[i], tau_abs) || bad(Drw[i], tw))) pi[j] = i;
        }
        /* fixes: a column-named error (i, j) whose row also names j is alone in row and column
         * (row formula); a column-named one whose row names something else shares its row
         * (column formula: the column holds only it); then row-named errors in columns that
         * named nothing (they share their column: row formula) */
        int nfix = 0;
        for (int j = 0; j < n; j++) {
            const int i = pi[j];
            if (i < 0) continue;
            const int jr = ratio_index(Drw[i], Dr[i], tau_abs, tw, n);
            const double d = (jr == j) ? fix_row(n, L, ldl, r, i, j) : fix_col(n, L, ldl, c, i, j);
            push_ev(rep, ORA_EV_FIX_DATA, panel, i, j, d);
            nfix++;
        }
        for (int i = 0; i < n; i++) {
            if (!bad(Dr[i], tau_abs)) continue;
            const int j = ratio_index(Drw[i], Dr[i], tau_abs, tw, n);
            if (j < 0 || !(bad(Dc[j], tau_abs) || bad(Dcw[j], tw)) || pi[j] >= 0) continue;
            const double d = fix_row(n, L, ldl, r, i, j);
            push_ev(rep, ORA_EV_FIX_DATA, panel, i, j, d);
            nfix++;
        }
        if (nfix == 0) break;
        }
        /* checksum words.  A data error flags both syndromes of its row in at least one sense and
         * its column likewise, so a word is refreshed only when the orthogonal direction shows
         * no flag of either kind anywhere (else: refuse at the re-verification) */
        for (int i = 0; i < n; i++) { Dr[i] = r[i] - row_e(n, L, ldl, i); Drw[i] = rw[i] - row_w(n, L, ldl, i); }
        for (int j = 0; j < n; j++) { Dc[j] = c[j] - col_e(n, L, ldl, j); Dcw[j] = cw[j] - col_w(n, L, ldl, j); }
        int anyR = 0, anyC = 0;
        for (int i = 0; i < n; i++) anyR |= bad(Dr[i], tau_abs) || bad(Drw[i], tw);
        for (int j = 0; j < n; j++) anyC |= bad(Dc[j], tau_abs) || bad(Dcw[j], tw);
        if (anyR && !anyC)
            for (int i = 0; i < n; i++) {
                if (bad(Dr[i], tau_abs)) {
                    const double old = r[i];
                    r[i] = row_e(n, L, ldl, i);
                    push_ev(rep, ORA_EV_FIX_R, panel, i, -1, r[i] - old);
                }
                if (bad(Drw[i], tw)) {
                    const double old = rw[i];
                    rw[i] = row_w(n, L, ldl, i);
                    push_ev(rep, ORA_EV_FIX_RW, panel, i, -1, rw[i] - old);
                }
            }
        if (anyC && !anyR)
            for (int j = 0; j < n; j++) {
                if (bad(Dc[j], tau_abs)) {
                    const double old = c[j];
                    c[j] = col_e(n, L, ldl, j);
                    push_ev(rep, ORA_EV_FIX_C, panel, -1, j, c[j] - old);
                }
                if (bad(Dcw[j], tw)) {
                    const double old = cw[j];
                    cw[j] = col_w(n, L, ldl, j);
                    push_ev(rep, ORA_EV_FIX_CW, panel, -1, j, cw[j] - old);
                }
            }
        /* kappa: both sums off by the same amount */
        {
            double sr = 0.0, sc = 0.0;
            for (int i = 0; i < n; i++) sr += r[i];
            for (int j = 0; j < n; j++) sc += c[j];
            if (!approx(sr, *kappa, tauS) && approx(sr, sc, tauS)) {
                const double old = *kappa;
                *kappa = sr;
                push_ev(rep, ORA_EV_FIX_K, panel, -1, -1, *kappa - old);
            }
        }
    }
    if (result == 1 || result == 0) {
        /* weighted words against the (verified / repaired) data: a weighted line that disagrees
         * while its plain line agrees is a corrupted weighted word (a data error with |d| <= tau
         * moves a weighted sum by at most n |d| <= tw) -- refresh it; corners likewise */
        int refreshed = 0;
        for (int i = 0; i < n; i++) {
            const double t = row_w(n, L, ldl, i);
            if (bad(rw[i] - t, tw) && !detected_here) {  /* v2 verified the data: a weighted word */
                const double old = rw[i];
                rw[i] = t;
                push_ev(rep, ORA_EV_FIX_RW, panel, i, -1, rw[i] - old);
                refreshed++;
            }
        }
        for (int j = 0; j < n; j++) {
            const double t = col_w(n, L, ldl, j);
            if (bad(cw[j] - t, tw) && !detected_here) {
                const double old = cw[j];
                cw[j] = t;
                push_ev(rep, ORA_EV_FIX_CW, panel, -1, j, cw[j] - old);
                refreshed++;
            }
        }
        double srw = 0.0, scw = 0.0;
        for (int i = 0; i < n; i++) srw += rw[i];
        for (int j = 0; j < n; j++) scw += cw[j];
        if (!approx(srw, *krw, twS)) {
            const double old = *krw;
            *krw = srw;
            push_ev(rep, ORA_EV_FIX_KW, panel, 0, -1, *krw - old);
            refreshed++;
        }
        if (!approx(scw, *kcw, twS)) {
            const double old = *kcw;
            *kcw = scw;
            push_ev(rep, ORA_EV_FIX_KW, panel, -1, 0, *kcw - old);
            refreshed++;
        }
        if (refreshed && result == 0) {
            push_ev(rep, ORA_EV_DETECT, panel, 0, 0, 0.0);
            if (rep) { rep->detected++; rep->corrected++; }
            result = 1;
        }
        /* final re-verification of all four syndromes and the corners */
        int ok = 1;
        double sr = 0.0, sc = 0.0;
        for (int i = 0; i < n && ok; i++) {
            ok &= !bad(r[i] - row_e(n, L, ldl, i), tau_abs) && !bad(rw[i] - row_w(n, L, ldl, i), tw);
            sr += r[i];
        }
        for (int j = 0; j < n && ok; j++) {
            ok &= !bad(c[j] - col_e(n, L, ldl, j), tau_abs) && !bad(cw[j] - col_w(n, L, ldl, j), tw);
            sc += c[j];
        }
        if (ok) ok = approx(sr, *kappa, tauS) && approx(sc, *kappa, tauS);
        if (!ok) {
            push_ev(rep, ORA_EV_UNCORRECTABLE, panel, -1, -1, 0.0);
            if (rep) rep->uncorrectable++;
            result = 2;
        } else if (detected_here && rep) {
            rep->corrected++;
        }
    }
    free(L0); free(r0); free(c0); free(Dr); free(Dc); free(Drw); free(Dcw); free(pi);
    return result;
}

/* encode (Fig. 3, Alg. 3 l.2): r = A e, c = e^T A, kappa = e^T A e (R22) */
void ora_encode(int n, const double *A, int lda, double *r, double *c, double *kappa) {
    row_sums(n, A, lda, r);
    for (int j = 0; j < n; j++) {
        double s = 0.0;
        for (int i = 0; i < n; i++) s += AT(A, lda, i, j);
        c[j] = s;
    }
    double k = 0.0;
    for (int i = 0; i < n; i++) k += r[i];
    *kappa = k;
}

/* ------------------------------------------------------------------ */
/* ABFT driver                                                          */
/* ------------------------------------------------------------------ */

/* logical H matrix (R6): stored Householder vectors of finished columns
 * (j in [ilo-1, cdone), i >= j+2) read as 0 */
static int is_v(int i, int j, int ilo, int ihi, int cdone) {
    return j >= ilo - 1 && j < cdone && j <= ihi - 2 && i >= j + 2 && i < ihi;
}

static void build_L(int n, const double *A, int lda, int ilo, int ihi, int cdone, double *L, int q) {
#pragma omp parallel for schedule(static)
    for (int j = 0; j < n; j++)
        for (int i = 0; i < n; i++) {
            int v = is_v(i, j, ilo, ihi, cdone);
            AT(L, n, i, j) = (q ? v : !v) ? AT(A, lda, i, j) : 0.0;
        }
}

static void write_back(int n, double *A, int lda, int ilo, int ihi, int cdone, const double *L, int q) {
    for (int j = 0; j < n; j++)
        for (int i = 0; i < n; i++) {
            int v = is_v(i, j, ilo, ihi, cdone);
            if (q ? v : !v) AT(A, lda, i, j) = AT(L, n, i, j);
        }
}

static void inject(const ora_fault *f, int n, double *A, int lda, chk_t *k, ora_report *rep) {
    double *p = NULL;
    switch (f->site) {
    case ORA_SITE_A: if (f->i >= 0 && f->i < n && f->j >= 0 && f->j < n) p = &AT(A, lda, f->i, f->j); break;
    case ORA_SITE_R: if (f->i >= 0 && f->i < n) p = &k->r[f->i]; break;
    case ORA_SITE_C: if (f->j >= 0 && f->j < n) p = &k->c[f->j]; break;
    case ORA_SITE_K: p = k->kap; break;
    case ORA_SITE_QR: if (f->i >= 0 && f->i < n) p = &k->qr[f->i]; break;
    case ORA_SITE_QC: if (f->j >= 0 && f->j < n) p = &k->qc[f->j]; break;
    case ORA_SITE_RW: if (k->rw && f->i >= 0 && f->i < n) p = &k->rw[f->i]; break;
    case ORA_SITE_CW: if (k->cw && f->j >= 0 && f->j < n) p = &k->cw[f->j]; break;
    }
    if (!p) return;
    double d = ora_flip(p, f->bit);
    push_ev(rep, ORA_EV_INJECT, f->panel, f->i, f->j, d);
}

static double frob(int n, const double *A, int lda) {
    double s = 0.0;
    for (int j = 0; j < n; j++)
        for (int i = 0; i < n; i++) s += AT(A, lda, i, j) * AT(A, lda, i, j);
    return sqrt(s);
}

int ora_ft_dgehd2(int n, int ilo, int ihi, double *A, int lda, double *tau,
                  int nb, double c_thr, const ora_fault *faults, int nfaults,
                  ora_report *rep, int stop_after_panel, double *chk_out) {
    return ora_ft_dgehd2_ex(n, ilo, ihi, A, lda, tau, nb, c_thr, 0, faults, nfaults, rep, stop_after_panel, chk_out);
}

int ora_ft_dgehd2_ex(int n, int ilo, int ihi, double *A, int lda, double *tau,
                     int nb, double c_thr, int weighted, const ora_fault *faults, int nfaults,
                     ora_report *rep, int stop_after_panel, double *chk_out) {
    int info = check_args(n, ilo, ihi, A, lda, tau);
    if (info) return info;
    if (nb < 1) return -7;
    if (c_thr <= 0.0) c_thr = 2.0;
    if (rep) memset(rep, 0, sizeof(*rep));
    for (int c = 0; c < n - 1; c++) tau[c] = 0.0;
    if (n == 0) return 0;

    size_t nn = (size_t)n;
    double *r = (double *)calloc(nn, 8), *cc = (double *)calloc(nn, 8);
    double *qr = (double *)calloc(nn, 8), *qc = (double *)calloc(nn, 8);
    double *y = (double *)calloc(nn, 8), *w = (double *)calloc(nn, 8);
    double *L = (double *)malloc(nn * nn * 8);
    double *Dr = (double *)malloc(nn * 8), *Dc = (double *)malloc(nn * 8);
    double kap = 0.0, qk = 0.0, krw = 0.0, kcw = 0.0;
    double *rw = weighted ? (double *)calloc(nn, 8) : NULL, *cw = weighted ? (double *)calloc(nn, 8) : NULL;
    chk_t k = {r, cc, &kap, qr, qc, &qk, rw, cw, &krw, &kcw};

    ora_encode(n, A, lda, r, cc, &kap);
    if (weighted) encode_w(n, A, lda, rw, cw, &krw, &kcw);
    double normF = frob(n, A, lda);              /* invariant under the similarity */
    double tau_abs = c_thr * n * EPS * normF;    /* R10 */
    double unit = n * EPS * (normF > 0 ? normF : 1.0);
    int result = 0;

    int c0 = ilo - 1, clast = ihi - 2;           /* reflector columns */
    for (int c = c0; c <= clast; c++) {
        if ((c - c0) % nb == 0) {
            int t = (c - c0) / nb;
            /* boundary t: inject, then verify / decode / correct (Alg. 3 l.12-15) */
            for (int f = 0; f < nfaults; f++)
                if (faults[f].panel == t) inject(&faults[f], n, A, lda, &k, rep);
            build_L(n, A, lda, ilo, ihi, c, L, 0);
            /* drift and the paper's scalar statistic (recorded; R11) */
            {
                double sr = 0.0, sc = 0.0, dmax = 0.0;
                syn_t s = {Dr, Dc, 0, 0};
                syndromes(n, L, n, r, cc, kap, &s);
                for (int i = 0; i < n; i++) { sr += r[i]; if (fabs(Dr[i]) > dmax) dmax = fabs(Dr[i]); }
                for (int j = 0; j < n; j++) { sc += cc[j]; if (fabs(Dc[j]) > dmax) dmax = fabs(Dc[j]); }
                if (rep) {
                    double ps = fabs(sr - sc) / (unit * sqrt((double)n));
                    if (ps > rep->paper_stat_max || ps != ps) rep->paper_stat_max = ps;
                    if (dmax / unit > rep->max_drift && dmax <= tau_abs) rep->max_drift = dmax / unit;
                }
            }
            int dres = weighted ? ora_decode_w(n, L, n, r, cc, &kap, rw, cw, &krw, &kcw, tau_abs, rep, t)
                                : ora_decode(n, L, n, r, cc, &kap, tau_abs, rep, t, ORA_MODE_H);
            if (dres == 2) { result = 1; goto out; }
            if (dres == 1) write_back(n, A, lda, ilo, ihi, c, L, 0);
        }
        tau[c] = reflector_step(n, ihi, A, lda, c, y, w, &k);
        if (stop_after_panel >= 0 && ((c + 1 - c0) % nb == 0 || c == clast) &&
            (c - c0) / nb == stop_after_panel) {
            if (chk_out) {
                memcpy(chk_out, r, nn * 8);
                memcpy(chk_out + n, cc, nn * 8);
                chk_out[2 * n] = kap;
                if (weighted) {  /* [.. | r_w | c_w | krw | kcw] */
                    memcpy(chk_out + 2 * n + 1, rw, nn * 8);
                    memcpy(chk_out + 3 * n + 1, cw, nn * 8);
                    chk_out[4 * n + 1] = krw;
                    chk_out[4 * n + 2] = kcw;
                }
            }
            goto out;
        }
    }
    /* end: inject AT_END faults, final H verification (a12) and Q verification */
    for (int f = 0; f < nfaults; f++)
        if (faults[f].panel == -1) inject(&faults[f], n, A, lda, &k, rep);
    {
        int cdone = clast + 1;
        build_L(n, A, lda, ilo, ihi, cdone, L, 0);
        int dres = weighted ? ora_decode_w(n, L, n, r, cc, &kap, rw, cw, &krw, &kcw, tau_abs, rep, -1)
                            : ora_decode(n, L, n, r, cc, &kap, tau_abs, rep, -1, ORA_MODE_H);
        if (dres == 2) { result = 1; goto out; }
        if (dres == 1) write_back(n, A, lda, ilo, ihi, cdone, L, 0);
        /* Q: logical matrix = stored Householder vectors only */
        build_L(n, A, lda, ilo, ihi, cdone, L, 1);
        double tauQ = c_thr * n * EPS * sqrt((double)n);
        dres = ora_decode(n, L, n, qr, qc, &qk, tauQ, rep, -1, ORA_MODE_Q);
        if (dres == 2) { result = 1; goto out; }
        if (dres == 1) write_back(n, A, lda, ilo, ihi, cdone, L, 1);
    }
out:
    free(r); free(cc); free(qr); free(qc); free(y); free(w); free(L); free(Dr); free(Dc); free(rw); free(cw);
    return result;
}
