/*
 * oracle.h -- plain, slow, obviously-correct CPU oracle for the ABFT
 * Householder Hessenberg reduction of Jia, Luszczek & Dongarra (IPDPSW 2016).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load liboracle.so.
 * The product path (libftgehrd.so) shares no code, header, table or helper
 * with this directory.
 *
 * Citations "P:N" are lines of the paper text; "R#" are the
 * readings listed in DESIGN.md (taken from SURVEY.md 8(c)).
 *
 * Conventions: 0-based indices, column-major, A(i,j) = A[i + j*lda].
 * ilo/ihi are LAPACK's 1-based arguments.  FP64 throughout, no BLAS,
 * no fast-math.  OpenMP only over disjoint output entries; every sum is a
 * sequential loop, so results are bitwise identical for any thread count.
 */
#ifndef ORACLE_H
#define ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* fault sites (R16) */
enum { ORA_SITE_A = 0,  /* working-array word A(i,j): H, trailing, or stored V */
       ORA_SITE_R = 1,  /* row-checksum r(i)            (P:224 Ar_chk)       */
       ORA_SITE_C = 2,  /* column-checksum c(j)         (P:224 Ac_chk)       */
       ORA_SITE_K = 3,  /* corner kappa = e^T L e       (R22)                */
       ORA_SITE_QR = 4, /* Q row checksum Qr(i)              */
       ORA_SITE_QC = 5, /* Q column checksum Qc(j)              */
       ORA_SITE_RW = 6, /* weighted row checksum r_w(i) (NEXT-1, w_i = i+1)   */
       ORA_SITE_CW = 7  /* weighted column checksum c_w(j)                     */ };

/* event kinds */
enum { ORA_EV_INJECT = 0, ORA_EV_DETECT = 1, ORA_EV_FIX_DATA = 2, ORA_EV_FIX_R = 3,
       ORA_EV_FIX_C = 4, ORA_EV_FIX_K = 5, ORA_EV_FIX_Q = 6, ORA_EV_FIX_QR = 7,
       ORA_EV_FIX_QC = 8, ORA_EV_FIX_QK = 9, ORA_EV_UNCORRECTABLE = 10,
       ORA_EV_FIX_RW = 11, ORA_EV_FIX_CW = 12, ORA_EV_FIX_KW = 13 };

/* decoder modes */
enum { ORA_MODE_H = 0, ORA_MODE_Q = 1 };

typedef struct {
    int32_t panel;   /* boundary t >= 0 (before panel t), or -1 = at the end */
    int32_t site;    /* ORA_SITE_* */
    int64_t i, j;    /* 0-based position (j ignored for R/QR, i for C/QC) */
    int32_t bit;     /* 0..63 of the binary64 word */
    int32_t pad;
} ora_fault;

typedef struct {
    int32_t kind, panel;
    int64_t i, j;
    double delta;    /* INJECT: new-old; FIX_*: new-old of the repaired word */
} ora_event;

#define ORA_MAX_EVENTS 1024
typedef struct {
    int32_t detected, corrected, uncorrectable, nevents;
    double max_drift;        /* max boundary |D| / (n eps ||A||_F), fault-free drift */
    double paper_stat_max;   /* max |sum r - sum c| / (n^1.5 eps ||A||_F) */
    ora_event ev[ORA_MAX_EVENTS];
} ora_report;

/* LAPACK DGEHD2 semantics.  Returns 0 or -argno. */
int ora_dgehd2(int n, int ilo, int ihi, double *A, int lda, double *tau);

/* LAPACK DORGHR semantics: explicit Q = H(ilo)...H(ihi-1).  Returns 0 or -argno. */
int ora_dorghr(int n, int ilo, int ihi, const double *A, int lda, const double *tau,
               double *Q, int ldq);

/* Unblocked reduction with naive checksum bookkeeping, boundary verification,
 * decoding/correction, fault injection and Q protection (Alg. 3 P:216 read at
 * reflector granularity, Theorem 1, Sec. IV-E/F P:266-278).
 * nb: boundary spacing (the GPU run's panel width); c_thr: threshold constant
 * (tau_abs = c_thr * n * eps * ||A||_F, R10).
 * stop_after_panel >= 0: return right after the last reflector of that panel,
 * A left in its working state and [r(0:n) | c(0:n) | kappa] written to chk_out.
 * Returns 0, 1 (uncorrectable) or -argno. */
int ora_ft_dgehd2(int n, int ilo, int ihi, double *A, int lda, double *tau,
                  int nb, double c_thr, const ora_fault *faults, int nfaults,
                  ora_report *rep, int stop_after_panel, double *chk_out);

/* The same with the weighted checksum pair (NEXT-1, w_i = i + 1) when weighted = 1: r_w = L w,
 * c_w = w^T L and the corners e^T L w, w^T L e ride through every reflector (Theorem 1 with w,
 * P:268-274) and the boundary decoder is ora_decode_w; chk_out then holds
 * [r | c | kappa | r_w | c_w | e^T L w | w^T L e] (4n + 3 doubles). */
int ora_ft_dgehd2_ex(int n, int ilo, int ihi, double *A, int lda, double *tau,
                     int nb, double c_thr, int weighted, const ora_fault *faults, int nfaults,
                     ora_report *rep, int stop_after_panel, double *chk_out);

/* Decoder v3 (weighted pair): v2 first; if it refuses, location by D_w / D = w_i on the weighted
 * syndromes; weighted checksum words refreshed; full re-verification.  0 / 1 / 2 as ora_decode. */
int ora_decode_w(int n, double *L, int ldl, double *r, double *c, double *kappa, double *rw, double *cw,
                 double *krw, double *kcw, double tau_abs, ora_report *rep, int panel);

/* The R12 decoder on a dense logical n x n matrix L (ldl), checksums r, c and
 * corner kappa, threshold tau_abs.  Repairs L/r/c/kappa in place.
 * Returns 0 = clean, 1 = corrected, 2 = uncorrectable. */
int ora_decode(int n, double *L, int ldl, double *r, double *c, double *kappa,
               double tau_abs, ora_report *rep, int panel, int mode);

/* encoding: r = A e, c = e^T A, kappa = e^T A e */
void ora_encode(int n, const double *A, int lda, double *r, double *c, double *kappa);

/* flip bit `bit` of *x, return new - old (may be inf/nan) */
double ora_flip(double *x, int bit);

int ora_num_threads(void);

#ifdef __cplusplus
}
#endif
#endif
