/*
 * ftgehrd.h -- C ABI of the B200-native ABFT Hessenberg reduction.
 *
 * Method: Jia, Luszczek, Dongarra, "Hessenberg Reduction with Transient Error
 * Resilience on GPU-Based Hybrid Architectures", IPDPSW 2016.  "P:N" below is
 * a line of that paper's text; "R#" a reading in DESIGN.md.
 *
 * All matrices are column-major FP64.  Pointers named d* are DEVICE pointers
 * (cudaMalloc / torch CUDA tensors) owned by the caller; the library never
 * frees them.  h* pointers are HOST pointers (pinned memory recommended).
 * Library workspace (augmented array, checkpoint, V/Y/T/W panels, checksum
 * vectors) is cached per device and released by ft_finalize().
 *
 * Return value (LAPACK style "info"):
 *    0                 success (possibly after correcting soft errors; see report)
 *   -i                 argument i is illegal (1 n, 2 ilo, 3 ihi, 4 A, 5 lda,
 *                      6 tau, 7 opts / an opts field, 8 Q, 9 ldq)
 *    FT_E_UNCORRECTABLE a detected discrepancy could not be decoded (R12);
 *                      A and tau are undefined, the report holds the events
 *    FT_E_CUDA / FT_E_NCCL / FT_E_NOMEM   runtime failures
 * Every call returns only after its stream has finished (info depends on the
 * device-side verification outcome).
 *
 * Threading: the workspace, cached CUDA graphs and counters are per device and
 * process-global, so every entry point holds one process-wide lock for the whole call:
 * calls from several host threads (on one device or several) are serialised by the
 * library, not run concurrently.
 */
#ifndef FTGEHRD_H
#define FTGEHRD_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define FT_E_UNCORRECTABLE 1
#define FT_E_CUDA 2
#define FT_E_NCCL 3
#define FT_E_NOMEM 4

/* Fault-injection phases within panel iteration t (Alg. 3):
 *   BEFORE_PANEL  start of iteration t, before its checkpoint (the paper's Fig. 2
 *                 "after iteration t-1, before iteration t")
 *   AFTER_PANEL   after the panel factorization (DLAHR2, Alg. 3 l.5-7), before the updates
 *   AFTER_RIGHT   after the right update (Alg. 3 l.8-10), before the left update (l.11)
 *   AFTER_UPDATE  after the left update, before the end-of-iteration check (l.12)
 *   AT_END        after the last iteration, before the final verification (panel ignored) */
enum { FT_PHASE_BEFORE_PANEL = 0, FT_PHASE_AFTER_PANEL = 1, FT_PHASE_AFTER_RIGHT = 2,
       FT_PHASE_AFTER_UPDATE = 3, FT_PHASE_AT_END = 4 };

/* Fault sites (failure model P:48-52; areas of Fig. 2a):
 *   A   working-array word A(i,j): area 1 (rows above the panel), area 2
 *       (trailing matrix), area 3 (finished Householder vectors) or finished H
 *   R   row-checksum r(i)        (Ar_chk)
 *   C   column-checksum c(j)     (Ac_chk)
 *   K   corner kappa = e^T L e   (R22)
 *   Y   panel workspace Y(i,j)   (j = column within the panel; R15)
 *   V   panel workspace V(i,j)   (the copy the updates read; R15)
 *   T   block-reflector factor T(i,j), 0 <= i, j < 64 (the nb x nb upper triangle is what the
 *       left update W' = T^T V^T A reads; R15 extended to T) */
/*   RW, CW  weighted checksum words r_w(i), c_w(j) (opts.weighted = 1, NEXT-1) */
enum { FT_SITE_A = 0, FT_SITE_R = 1, FT_SITE_C = 2, FT_SITE_K = 3, FT_SITE_Y = 4, FT_SITE_V = 5, FT_SITE_T = 6,
       FT_SITE_RW = 7, FT_SITE_CW = 8 };

typedef struct {
    int32_t panel;  /* iteration t >= 0 (ignored for AT_END) */
    int32_t phase;  /* FT_PHASE_* */
    int32_t site;   /* FT_SITE_* */
    int32_t bit;    /* 0..63: XOR this bit of the binary64 word */
    int64_t i, j;   /* 0-based position (j unused for R, i unused for C) */
} ft_fault;

enum { FT_EV_INJECT = 0, FT_EV_DETECT = 1, FT_EV_FIX_DATA = 2, FT_EV_FIX_R = 3, FT_EV_FIX_C = 4,
       FT_EV_FIX_K = 5, FT_EV_FIX_Q = 6, FT_EV_FIX_QR = 7, FT_EV_FIX_QC = 8, FT_EV_FIX_QK = 9,
       FT_EV_UNCORRECTABLE = 10, FT_EV_ROLLBACK = 11, FT_EV_PANEL_REDO = 12,
       FT_EV_FIX_RW = 13, FT_EV_FIX_CW = 14, FT_EV_FIX_KW = 15 /* weighted pair words (NEXT-1) */ };

typedef struct {
    int32_t kind, panel;  /* FT_EV_*, iteration (-1 = final verification) */
    int64_t i, j;         /* position (DETECT: i = #flagged rows, j = #flagged cols) */
    double delta;         /* INJECT: new - old; FIX_*: repaired - corrupted */
} ft_event;

#define FT_MAX_EVENTS 256
typedef struct {
    int32_t detected, corrected, rollbacks, panel_redos, uncorrectable, nevents;
    double max_drift_rel;       /* max |maintained - recomputed| / (n eps ||A||_F) seen */
    double ms[8];               /* device ms (CUDA events on the call's stream): 0 the whole call;
                                   with opts.timing = 1 the phases 1 panel (DLAHR2 kernel + Y_top),
                                   2 right update (+ W), 3 left update, 4 separate verification
                                   launches (unfused checks, final verification; fused checks are
                                   inside 1-3), 5 recovery (rollback, restore, locate, correct),
                                   6 copy-in/out, 7 encode; -1 when opts.timing = 0 */
    ft_event events[FT_MAX_EVENTS];
} ft_report;

enum { FT_POLICY_EAGER = 0, FT_POLICY_PAPER = 1 };

typedef struct {
    int32_t nb;          /* panel width; 0 -> 32 if n < 4096 else 64 (R4); max 64      */
    int32_t abft;        /* 0 = fault-prone baseline (no checksums), 1 = protected     */
    int32_t weighted;    /* 1 (with abft = 1): + the weighted checksum pair r_w = L w, c_w = w^T L,
                            w_i = i + 1 (NEXT-1), riding as row / column n+1 through every update;
                            the decoder then locates tied and L-shaped multiple errors;
                            the stop hook's dchk_out holds 4n+3 doubles
                            [r | c | kappa | r_w | c_w | e^T L w | w^T L e]                     */
    int32_t policy;      /* FT_POLICY_EAGER (default) or FT_POLICY_PAPER (R11)         */
    double c_thr;        /* threshold constant; 0 -> 2.0; tau_abs = c_thr*n*eps*||A||_F (R10) */
    const ft_fault *faults;   /* host array, may be NULL                                 */
    int32_t nfaults;
    ft_report *report;        /* optional host output                                    */
    int32_t stop_after_panel; /* verify hook: -1 = run to the end; t >= 0 = stop after
                                 iteration t, copy the WORKING matrix (H/V so far, trailing
                                 part updated) to dA and the maintained checksums
                                 [r(0:n) | c(0:n) | kappa] to dchk_out                   */
    double *dchk_out;         /* device buffer of 2n+1 doubles, or NULL                  */
    void *stream;             /* cudaStream_t; NULL -> the legacy default stream          */
    int32_t timing;           /* 1: record the per-phase times report->ms[1..7] (an event pair
                                 around each phase; such calls are never graph-replayed)     */
    int32_t deterministic;    /* 1: bitwise reproducible results -- the panel's cross-CTA column
                                 dots are summed in a fixed order (each CTA stores its partial,
                                 every CTA sums them after the grid barrier) instead of by FP64
                                 atomics, so two identical calls (and the ranks of a multi-GPU
                                 call) give bitwise-equal H, tau, Q; costs one L2 round trip
                                 per column reduction                          */
} ft_opts;

/* Fill *o with defaults (nb 0, abft 1, policy EAGER, c_thr 2, no faults, run to end). */
void ft_opts_default(ft_opts *o);

/* Reduce A to upper Hessenberg form H = Q^T A Q (LAPACK DGEHRD semantics, P:38-42,
 * Alg. 3).  On exit H is on and above the first subdiagonal of dA and the
 * Householder vectors v(i+2:ihi) of H(i) = I - tau(i) v v^T are stored below it
 * (v(i+1) = 1 implicit).  dtau has n-1 entries; tau(1:ilo-1) = tau(ihi:n-1) = 0.
 * 1 <= ilo <= ihi <= n (n = 0: ilo = 1, ihi = 0); A is assumed upper triangular
 * in rows/columns 1:ilo-1 and ihi+1:n.  lda >= max(1, n). */
int ft_dgehrd(int n, int ilo, int ihi, double *dA, int lda, double *dtau, const ft_opts *opts);

/* NEXT-4 (the paper's generalisation claim): symmetric tridiagonal reduction A = Q T Q^T with
 * LAPACK DSYTRD semantics for uplo = 'L', on the protected path.  For symmetric A the Householder
 * Hessenberg reduction IS the tridiagonal reduction (same reflectors, same DLARFG convention: H is
 * tridiagonal, v(i+2:n) of H(i) stored below the subdiagonal), so the call runs ft_dgehrd's ABFT
 * machinery (checksums, verification, rollback, correction, fault plan) on the symmetric matrix the
 * lower triangle of dA defines (the strict upper triangle is not referenced).  It does not exploit the
 * symmetry (no SYMV / SYR2K: about 2.5x the flops of a symmetric-specific code).  On exit: d (n) the
 * diagonal, e (n-1) the subdiagonal of T, tau (n-1), V below the subdiagonal of dA; Q by ft_dorghr.
 * Device pointers; errors as ft_dgehrd (-4 d, -5 e / lda, -6 tau). */
int ft_dsytrd(int n, double *dA, int lda, double *dd, double *de, double *dtau, const ft_opts *opts);

/* Same contract with HOST buffers hA / htau: the host->device copy of A, the
 * reduction and the device->host copy of H/V and tau all run inside the call
 * (the end-to-end entry point bench.py times). */
int ft_dgehrd_host(int n, int ilo, int ihi, double *hA, int lda, double *htau, const ft_opts *opts);

/* Form the explicit orthogonal Q = H(ilo) H(ilo+1) ... H(ihi-1) (Q = Q1 Q2 ... Qn-1) from the
 * output of ft_dgehrd (LAPACK DORGHR semantics; Q is the identity outside rows/cols ilo..ihi and
 * Q e1 = e1 when ilo = 1).  dQ may alias dA only if ldq == lda.  Blocked and backward: panel
 * t = npanels-1 .. 0 (columns k = ilo-1 + t nb ..) applies Q = (I - V T V^T) Q with the DMMA kernels.
 * opts NULL: the plain formation.  opts->abft = 1 (NEXT-3): checksum-protected accumulation -- Q
 * carries a row checksum r = Q e, a column checksum c = e^T Q and kappa through every update
 * (Theorem 1), each iteration ends with the sum check (rolled back and located on a
 * mismatch), and Q is verified and corrected at the end (R12 decoder).  Read: nb, abft,
 * c_thr, faults (sites A = Q(i,j), R, C, K of Q's checksums; phases BEFORE_PANEL / AFTER_UPDATE of
 * panel t, AT_END), report, stream, timing.  Returns 0, FT_E_UNCORRECTABLE (Q undefined), or the
 * argument / runtime codes of ft_dgehrd (-8 dQ, -9 ldq). */
int ft_dorghr(int n, int ilo, int ihi, const double *dA, int lda, const double *dtau,
              double *dQ, int ldq, const ft_opts *opts);

/* ---------------------------------------------------------------------------------
 * Multi-GPU reduction (the north star's "1-D block-column cyclic across
 * 2/4/8 B200").  Layout: global column J (0-based) lives on rank (J / nb) mod nranks at
 * local column (J / (nb * nranks)) * nb + J mod nb, nb = opts->nb (0 -> 32 if n < 4096
 * else 64); each rank passes its n x ncols_local slab (column-major, lda_local >= n).
 * Every rank runs the DLAHR2 panel redundantly on a broadcast copy of the panel columns;
 * the trailing GEMV of every column covers only the rank's own columns and its partial
 * sums are exchanged CTA by CTA through peer memory inside the persistent panel kernel
 * (no host collective per column); Y_top is a per-rank partial summed by a peer
 * allreduce; the block-reflector updates are rank-local.  tau is replicated on return.
 * Scope: ilo = 1, ihi = n, no stop hook (-2 / -3 / -7 otherwise).  With abft = 1 the checksums
 * ride through every update (r replicated, c with its columns); every iteration ends with the
 * paper's sum check on rank-ordered allreduced sums, so every rank halts identically;
 * the iteration is then added back (reverse computation), the checkpoint restored, the error
 * located from the summed row sums and the gathered column discrepancies, and repaired by the
 * owner of its column (R12 decoder); the finished H is verified and corrected at the end.
 * Fault plans: sites A and C (j = the GLOBAL column; the owner's word) at BEFORE_PANEL,
 * AFTER_RIGHT, AFTER_UPDATE and AT_END (-7 for the replicated r / kappa and the per-rank
 * V, Y, T copies, and for AFTER_PANEL).
 *
 * Bootstrap (one process per GPU): ft_mgpu_setup allocates this rank's workspace,
 * including a peer-visible region, for matrices up to n_max and returns its CUDA IPC
 * handle; the caller all-gathers the handles (e.g. torch.distributed) and passes them to
 * ft_mgpu_connect, which maps every peer's region.  Errors: -9 bad rank / nranks /
 * call order, FT_E_CUDA / FT_E_NOMEM as for ft_dgehrd.  All ranks must issue the same
 * sequence of ft_dgehrd_mgpu calls (same n, nb, abft). */
typedef struct { char bytes[64]; } ft_ipc_handle;
int ft_mgpu_setup(int n_max, int rank, int nranks, ft_ipc_handle *handle_out);
int ft_mgpu_connect(const ft_ipc_handle *handles, int rank, int nranks);
int ft_dgehrd_mgpu(int n, int ilo, int ihi, double *dA_local, int lda_local, double *dtau,
                   int rank, int nranks, const ft_opts *opts);

/* The same sharded reduction with nranks VIRTUAL ranks on the current GPU (one process):
 * dA_local[q] / dtau[q] are rank q's slab and tau (device pointers, q < nranks <= 8).
 * Identical kernels and exchange protocol; the ranks' CTA groups share one cooperative
 * launch and reach each other's buffers through plain device pointers.  Used to test and
 * measure the multi-GPU path on one GPU. */
int ft_dgehrd_vranks(int n, int ilo, int ihi, double *const *dA_local, int lda_local,
                     double *const *dtau, int nranks, const ft_opts *opts);

/* Bootstrap probe of the IPC mappings (no kernel): ft_mgpu_probe_put(v) writes v into slot `rank` of
 * every rank's symmetric region through the peer mappings (ordinary copies); after a barrier between
 * the processes, ft_mgpu_probe_get(out) reads this rank's nranks slots.  -9 before setup/connect. */
int ft_mgpu_probe_put(double v);
int ft_mgpu_probe_get(double *out);

/* Release the multi-rank workspaces (virtual ranks and this process's rank). */
void ft_mgpu_finalize(void);

/* Human-readable text for an info code. */
const char *ft_strerror(int info);

/* Release all cached device workspace. */
void ft_finalize(void);

/* Library build / capability string (arch, version). */
const char *ft_version(void);

/* Kernel-launch counter (for the bench's gpu_launches claim): number of kernels this
 * library has launched since load / the last reset. */
int64_t ft_launch_count(int reset);

/* Diagnostics (used by bench.py for the roofline of the dominant kernel).
 * ft_debug_time_panels(1) resets and starts recording CUDA events around every panel
 * kernel launch on its stream; ft_debug_panel_ms() / ft_debug_panel_launches() return the
 * summed device time and launch count of completed calls.  ft_debug_probe_panel(t, dbuf)
 * makes CTA 0 of panel t write per-column phase timestamps (clock64, 16 slots per column at
 * [j*16], the max over CTAs of each phase at [1024 + j*16]; the wide kernel's per-CTA GEMV spans
 * at [2048 + 4*cta]; CTA 0's kernel entry / epilogue end at [3072] / [3073]: a device buffer of
 * 3088 uint64) -- t = -1 disables. */
void ft_debug_time_panels(int on);
double ft_debug_panel_ms(void);
int ft_debug_panel_launches(void);
/* The same for the bench's kernel classes cls = 0 panel kernel, 1 right-update launch (+ W),
 * 2 left-update launch: ft_debug_time_kernels(1) resets and starts (graph replay off while on). */
void ft_debug_time_kernels(int on);
double ft_debug_kernel_ms(int cls);
int ft_debug_kernel_launches(int cls);
void ft_debug_probe_panel(int panel, unsigned long long *dbuf);
/* ft_debug_panel_path(8) sends every column of every later panel through the explicit
 * two-reduction path (the one-reduction path's cancellation fallback); 64 / 128 force the
 * panel's smaller shared-memory modes (V, Z rows cached, Y global / all global); 0 restores
 * the default.  Results agree with the default up to rounding (tests of those paths). */
void ft_debug_panel_path(int bits);
/* ft_debug_left_fold(0) makes the ABFT left update carry the checksum row c and column r as
 * an extra DMMA tile row / column strip (the round-1 layout) instead of folding them into
 * the CTAs of the last tile row / strip (1, the default).  Results agree
 * up to rounding; CUDA-graph replay is off while 0. */
void ft_debug_left_fold(int on);
/* ft_debug_right_fold(0) makes the ABFT right update carry the column checksum c (row n) as one
 * more DMMA tile row instead of a GEMV by the CTAs of the last row split (1, the default; the
 * row splits then see the data rows only).  Results agree up to rounding; CUDA-graph replay is
 * off while 0. */
void ft_debug_right_fold(int on);
/* Number of panel launches that ran the two-reduction wide kernel (>= 32 rows per CTA, the large-n
 * path) since load / the last reset: tests use it to show which panel kernel a run exercised. */
int64_t ft_debug_wide_launches(int reset);
/* Host-side diagnostics of the right update's row-split model (no device work): the number of row
 * splits chosen for the block rows [r_lo, r_hi) x columns [c_lo, c_hi) on nsm SMs (extra_strips:
 * the M-part strip; wr_lo: the first row of the W pass, -1 for none), and the tile range [t0, t1)
 * that split y of ns gets when a strip of nrt tiles has tw right-only tiles at the top (weights 1
 * and 2: the splits cut the strip into equal weights). */
int ft_debug_right_splits(int r_lo, int r_hi, int c_lo, int c_hi, int nsm, int extra_strips, int wr_lo);
void ft_debug_right_split_range(int nrt, int tw, int ns, int y, int *t0, int *t1);

#ifdef __cplusplus
}
#endif
#endif
