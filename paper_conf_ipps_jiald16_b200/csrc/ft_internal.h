// ft_internal.h -- internal structures and kernel launchers of libftgehrd.
// Host + device visible; no torch types, no oracle code.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/ftgehrd.h"

#define FT_MAXFAULTS 64
#define FT_MAX_VRANKS 8      // ranks per multi-rank launch (virtual ranks on one GPU) / max ranks
#define FT_FLAG_STRIDE 256   // per-rank stride of the exchange flag arrays (>= CTAs per rank)
#ifndef FT_NBMAX
#define FT_NBMAX 64
#endif
#define FT_ESTR 4  // doubles per pre-update check sum (FtCtl::eY / eV)
#define FT_ACC_STRIDE (3 * 64 + 8)  // [s1 | sx | scalars | V^T x] per reduction set (ft_panel.cu ACC_*)
#define FT_ACC_SETS 4               // sets indexed by the global column mod 4 (recycled in-kernel)
#define FT_ACC_PAD 32               // doubles between accumulators: one 256-byte block (own L2 slice) each
#define FT_ACC_SET_DOUBLES (FT_ACC_STRIDE * FT_ACC_PAD)
#ifndef FT_DPMAX
#define FT_DPMAX 160  // deterministic mode: max CTAs per panel launch (rank group)
#endif

// Device-resident control block: halt protocol, fused-verify flags, injector log.
struct FtCtl {
    int halt;         // != 0: every later kernel of this call is a no-op
    int halt_panel;   // iteration at which the halt was raised
    int halt_stage;   // 1 = pre-update (verify-before-consume / workspace check), 2 = post-update,
                      // 3 = T checksum failed after the right update (only the right update to undo)
    int halt_reason;  // bit 0: D_r flag, 1: Y check, 2: V check, 3: scalar check (paper), 4: kappa, 5: T check,
                      // 6: weighted sums (NEXT-1)
    int nflag;        // flagged rows in the fused verify of the current iteration
    int done_count;   // last-block-done counter (k_endcheck)
    int done_ytop;    // last-block-done counter (fused pre-update decision in the Y_top finalize)
    int done_left;    // last-CTA-done counter (fused end-of-iteration check in the left update)
    double normF;         // ||A||_F of the input (invariant under the similarity)
    double c_thr;
    unsigned long long drift_bits;  // max fault-free |D| / (n eps ||A||_F) seen (as bits)
    // pre-update check sums e^T Y, e^T V of column j at [j * FT_ESTR]: one 32-byte sector per
    // column, so the per-CTA atomics of different columns do not serialise on shared sectors
    double eY[64 * FT_ESTR];
    double eV[64 * FT_ESTR];
    double sums[4];       // end check: sum r, sum c
    double wsums[2];      // end check of the weighted pair: sum r_w, sum c_w (NEXT-1)
    double tmax;          // max |T| of the last panel (written by the panel kernel; pre-update tolerance)
    // T checksum (reading R15 extended to T): row sums of the upper triangle of the panel's T, written
    // by the panel kernel with T; re-evaluated from T in memory by the right-update CTAs that form
    // W' = T^T W.  A mismatch sets tbad (the right update has then been applied in full); the left
    // update launch turns it into a halt of stage 3 (roll back the right update, redo the panel)
    double tchk[64];
    int tbad;
    int fflag;  // device-side final verification: bit 0 H, bit 1 Q needs the host decoder
    double inj_delta[FT_MAXFAULTS];
    int inj_done[FT_MAXFAULTS];
};

struct PanelParams {
    double *A;
    int64_t ldw;
    double *V, *Y, *T, *tau, *acc;
    // deterministic mode (opts.deterministic): the column dots' CTA partials are stored, not added,
    // at dpart[(set * FT_ACC_STRIDE + i) * FT_DPMAX + cta] and summed in a fixed order after the grid
    // barrier (ft_common.cuh det_sum): bitwise reproducible panels.  NULL: FP64 atomics into acc
    double *dpart;
    double *bvec;        // [4][ldw]: b0 of columns c (parity c & 1), x of the explicit path (2 + parity)
    double *Z;           // ldw x FT_NBMAX: A(:, c+2:) V_x of the own rows when they do not fit in smem
    unsigned *bar;       // grid-barrier counter of this launch (zero at launch)
    unsigned *bar_next;  // the next panel launch's counter (zeroed by this launch)
    FtCtl *ctl;
    double *Qr, *Qc;
    int n, ihi, k, ib, abft, verify;  // verify: fused D_r on the first GEMV (EAGER policy)
    int rbase, ngroups;               // ft_panel_group_rows()-row groups starting at rbase
    int wide;                         // set by the launcher: >= 32 rows per CTA (GEMV on 15 warps)
    int ytop;                         // rows 0..k ride along (rbase = 0): Y_top and the M-part by the panel
    int ncc;                          // set by the launcher: trailing columns whose row slabs live in smem
    // diskless checkpoint of the panel, taken in the kernel's prologue, or NULL
    double *ckpt, *ck_r, *ck_c, *ck_q, *Fr;
    int precheck_sums;  // add e^T Y, e^T V of the own rows into ctl->eY / eV (fused pre-update check)
    // deferred end check of the previous iteration (left update with endcheck = 2): every CTA
    // reads ctl->sums[2:4] and kappa at entry, with the halt flag, and compares them before its
    // first store (EAGER: sum r and sum c against kappa; PAPER: with each other); a failure
    // raises the halt for panel echeck_panel (stage 2) and the launch does nothing.  CTA 0 clears
    // the sums after the first grid barrier.
    int echeck, echeck_panel, echeck_policy;
    unsigned long long *dbg;          // optional per-column phase timestamps (CTA 0), or NULL
    int dbg_mode;                     // timing ablations (wrong results): 1 no grid barriers, 2 no GEMV, 4 no atomics;
                                      // 8: every column on the explicit (two-reduction) path (exact)
    // panel columns: Apan[row + c * ldw] is panel column c (k <= c < k + ib); == A on one GPU.
    // rcol: the row-checksum column r.
    double *Apan, *rcol;
    // multi-rank mode (1-D block-column cyclic); G == 1 on one GPU.  A is the
    // rank's local slab: local column l holds global column J(l) = (l / cbnb) G cbnb +
    // rank cbnb + l % cbnb.  The trailing GEMV covers the panel columns (owner only, from
    // Apan) and the local columns [lcol0, lcol1) (global >= e); the per-column GEMV
    // partials are exchanged through peer memory, CTA by CTA (no collective, no host).
    int G, rank, cbnb, owner, lcol0, lcol1, e;
    double2 *yx;                     // own exchange slots [2][G][ldw]: (y partial, A(:, c+1) part)
    double2 *ypeer[FT_MAX_VRANKS];   // every rank's slot base (index = rank; own included)
    unsigned *flags;                 // own arrival flags [G][FT_FLAG_STRIDE]
    unsigned *fpeer[FT_MAX_VRANKS];  // every rank's flag array
    unsigned seq0;                   // flag value of column c is seq0 + c + 1
};
// A multi-rank launch: nr ranks (virtual ranks sharing this GPU, or 1 per GPU), each a
// group of gridDim.x / nr CTAs with identical row partitions.
struct PanelLaunch {
    PanelParams r[FT_MAX_VRANKS];
    int nr;
};

// launchers (return cudaError_t of the launch)
cudaError_t ft_launch_panel(const PanelParams &p, int nsm, cudaStream_t s);
cudaError_t ft_launch_panel_multi(const PanelLaunch &L, int nsm, cudaStream_t s);
cudaError_t ft_launch_panel_wide(const PanelLaunch &L, int nsm, cudaStream_t s);  // two-reduction kernel
size_t ft_panel_smem_bytes();
int ft_panel_group_rows();
int ft_panel_cta_cap();  // FT_PANEL_CTAS experiment cap on the panel grid (0: none)

struct GemmRightParams {
    double *A;
    int64_t lda;    // leading dimension of A (the updated matrix)
    int64_t ldw;    // leading dimension of Y and V
    const double *Y, *V;
    int r_lo, r_hi, c_lo, c_hi, K;  // C rows/cols, inner dimension
    int wr_lo, wr_hi;               // rows of V that take part in W = V^T A_new
    int do_right, do_w;
    double sign;                    // -1: A -= Y V^T (update), +1: rollback
    double *Wpart;                  // W partials [split][col][64] (one per row split, no atomics)
    int64_t wsplit_stride;          // doubles per split
    int nsplit;                     // row splits (grid.y); use ft_gemm_splits()
    const FtCtl *ctl;
    // optional M-part (DGEHRD's DTRMM + DAXPY on rows 0..m_r_hi-1 of columns m_c_lo..m_c_hi-1),
    // run as one extra strip of the same launch (no W)
    int has_m, m_c_lo, m_c_hi, m_r_hi;
    // W' = op(T) W formed by the last CTA of each strip (the left update's operand), if Wt != NULL
    double *Wt;
    const double *T;
    int transT;
    int *strip_done;  // per-strip arrival counters (zero; reset by their last CTA)
    // multi-rank column map: local column l of A is global column
    // ft_cmap(l) (the row of V it pairs with); cm_G <= 1 is the identity
    int cm_G, cm_rank, cm_nb, cm_ncl, cm_n;
    // fused pre-update check (reading R15, EAGER): every CTA evaluates e^T Y = Y_chk, e^T V = V_chk
    // and the fused D_r flag count before touching A; a failed check halts the whole launch
    FtCtl *pre_ctl;  // non-NULL: evaluate the check (pre_n, pre_panel)
    int pre_n, pre_panel;
    // T checksum check (ABFT): the last CTA of each strip verifies the T it read against ctl->tchk
    // before forming W' = op(T) W; on a mismatch it sets ctl->tbad (non-NULL: check on)
    FtCtl *tctl;
    // fold (ABFT, single rank): the column-checksum row c = row r_hi-1 (= n) is not a tile row;
    // the CTAs of the last row split update it as a GEMV c(cols) += sign Y(n, :) V(cols, :)^T
    // (kappa with the column-n strip), so a whole 64-row tile is not spent on one row and the row
    // splits see the data rows only (nsplit: ft_gemm_splits over [r_lo, r_hi-1))
    int fold_row;
};
// global column of local column l in the 1-D block-column cyclic layout; local column ncl
// is the replicated row-checksum column r (global n)
__host__ __device__ inline int ft_cmap(int l, int G, int rank, int nb, int ncl, int n) {
    if (G <= 1) return l;
    if (l == ncl) return n;
    return (l / nb) * nb * G + rank * nb + l % nb;
}
cudaError_t ft_launch_gemm_right(const GemmRightParams &p, cudaStream_t s);
struct CUtensorMap_st;
// 2-D TMA map of a column-major ldw x K panel, box rows x K (ft_gemm.cu); 0 on success
int ft_panel_tmap(struct CUtensorMap_st *m, const double *base, int64_t ldw, int K, int rows);
#define FT_WSPLIT_MAX 32  // max row splits of the right update (deterministic W partials)
// row splits the right-update launch uses for this block (the left update's k_wprep sums them)
// wr_lo: first row of the W pass (tiles above it are weighted as right-only, see ft_gemm.cu); -1: all
int ft_gemm_splits(int r_lo, int r_hi, int c_lo, int c_hi, int nsm, int extra_strips = 0, int wr_lo = -1);

struct GemmLeftParams {
    double *A;
    int64_t lda;
    int64_t ldw;
    const double *V, *T, *Wpart;  // Wpart: the right update's W partials [split][col][64]
    double *Wt;                     // scratch for W' = op(T) W ([col][64])
    int r_lo, r_hi, c_lo, c_hi, K;
    int nsplit;     // number of W partials to sum (the right update's splits)
    int64_t wsplit_stride;
    int transT;     // 1: A -= V (T^T W) (DLARFB 'L','T'); 0: A -= V (T W)
    double sign;    // -1 update, +1 rollback
    const FtCtl *ctl;
    int wt_ready;   // 1: Wt already holds op(T) W (formed by the right-update launch)
    // end-of-iteration check (Alg. 3 l.12-13) + frozen row sums: endcheck 1 = fused, the last CTA
    // decides; 2 = the partial sums only (the next panel launch decides, PanelParams::echeck)
    int endcheck, panel, policy, n;
    double *Fr;
    FtCtl *ectl;
    FtCtl *pre_reset;  // non-NULL: CTA (0,0) clears the fused pre-update sums for the next panel
    FtCtl *tctl;       // non-NULL: a set tctl->tbad (T checksum failed in the right update) makes the
                       // launch a no-op and raises the halt (stage 3) instead
    // 1: row r_hi-1 and column c_hi-1 are the checksum row c and column r (= n, ABFT); they are
    // updated by CUDA-core dot products in the CTAs owning the last row tile / column strip
    // instead of as an extra 64-row tile and 64-column strip of DMMA work (n % 64 == 0 would
    // otherwise add a whole strip and tile row for one column / one row)
    int fold;
    int ny, nyf;  // set by the launcher: CTA rows [0, nyf) form the frozen row sums, the next ny own tiles
};
cudaError_t ft_launch_gemm_left(const GemmLeftParams &p, cudaStream_t s);

struct YtopParams {
    const double *A;
    int64_t ldw;
    const double *V, *T;
    double *Y;
    double *ypart, *rowpart;  // [split][row][64], [split][row]
    const double *Fr;
    FtCtl *ctl;
    int n, ihi, k, ib, nsplit, abft, verify;
    int decide;  // fused pre-update check (R15): add e^T Y of rows 0..k, last block decides
    int panel;
    // multi-rank: the inner dimension runs over the local columns [kc0, kc1) (global >= k+1),
    // V rows through the column map; Y(0:k+1, :) is then this rank's partial
    int cm_G, cm_rank, cm_nb, cm_ncl, kc0, kc1;
};
int ft_ytop_rows_per_cta();  // rows of A per Y_top partial CTA (split sizing)
cudaError_t ft_launch_ytop(const YtopParams &p, cudaStream_t s);

// ABFT / utility kernels (ft_abft.cu)
cudaError_t ft_ctl_init(FtCtl *ctl, double c_thr, cudaStream_t s);
cudaError_t ft_copy_in(const double *A, int lda, double *Aw, int64_t ldw, int n, cudaStream_t s);
cudaError_t ft_copy_out(const double *Aw, int64_t ldw, double *A, int lda, int n, cudaStream_t s);
cudaError_t ft_mirror_lower(double *Aw, int64_t ldw, int n, cudaStream_t s);
cudaError_t ft_copy_out_lower(const double *Aw, int64_t ldw, double *A, int lda, int n, double *d, double *e,
                              cudaStream_t s);
cudaError_t ft_encode(double *Aw, int64_t ldw, int n, FtCtl *ctl, double *scratch, double *linepart,
                      cudaStream_t s);
cudaError_t ft_frozen_init(const double *Aw, int64_t ldw, int n, int ncols, double *Fr, cudaStream_t s);
cudaError_t ft_precheck(const double *Y, const double *V, int64_t ldw, int n, int ihi, int k, int ib,
                        FtCtl *ctl, cudaStream_t s);
cudaError_t ft_decide(const double *Y, const double *V, const double *T, int64_t ldw, int n, int k,
                      int ib, int panel, FtCtl *ctl, cudaStream_t s);
cudaError_t ft_endcheck(double *Aw, int64_t ldw, int n, int ihi, int k, int ib, int panel, int policy,
                        double *Fr, FtCtl *ctl, cudaStream_t s, int weighted = 0);
cudaError_t ft_zero_if_running(double *p, size_t n, const FtCtl *ctl, cudaStream_t s);
cudaError_t ft_inject(double *addr, int fidx, int bit, FtCtl *ctl, cudaStream_t s);
// full verification (recovery path / final): mode 0 = H logical, 1 = Q (V region)
cudaError_t ft_full_verify(const double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode,
                           const double *r, int64_t rinc, const double *c, int64_t cinc, const double *Fr,
                           double *Dr, double *Dc, double *sums, double *linepart, cudaStream_t s);
// kind: 0 row formula, 1 col formula, 2 refresh r(i), 3 refresh c(j), 4 kappa; weighted pair (NEXT-1):
// 5 refresh r_w(i), 6 refresh c_w(j), 7 e^T L w = sum r_w, 8 w^T L e = sum c_w
struct FtFix { int64_t i, j; int kind; int pad; };
cudaError_t ft_encode_w(double *Aw, int64_t ldw, int n, double *linepart, cudaStream_t s);
// R12 decoder v2 on the device (one block): status 0 clean, 1 fixes planned, 2 uncorrectable, 3 the plan
// exceeds cap (the host decides)
struct FtDecOut { int status, nfix, nR, nC; };
cudaError_t ft_decode(const double *Dr, const double *Dc, const double *sums, const double *kap, int n, int mode,
                      const FtCtl *ctl, int *idx, FtFix *fixes, int cap, FtDecOut *out, cudaStream_t s);
cudaError_t ft_apply_fixes_dev(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode, double *r,
                               int64_t rinc, double *c, int64_t cinc, double *kappa, const FtFix *fixes, int cap,
                               double *deltas, const FtDecOut *dec, cudaStream_t s);
cudaError_t ft_final_flags(const double *Dr, const double *Dc, const double *sums, const double *kap, int n, int mode,
                           FtCtl *ctl, cudaStream_t s);
cudaError_t ft_full_verify_w(const double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, const double *rw,
                             const double *cw, int64_t cinc, double *Drw, double *Dcw, double *linepart,
                             cudaStream_t s);
cudaError_t ft_wchk(const double *Aw, double *V, double *Y, const double *T, int64_t ldw, int n, int ihi, int k,
                    int ib, double *part, const FtCtl *ctl, cudaStream_t s);
cudaError_t ft_cw_panel(double *Aw, int64_t ldw, int n, int ilo, int ihi, int k, int e, const FtCtl *ctl,
                        cudaStream_t s);
cudaError_t ft_ckpt_w(double *Aw, int64_t ldw, int n, double *ck, int restore, const FtCtl *ctl, cudaStream_t s);
cudaError_t ft_apply_fixes(double *Aw, int64_t ldw, int n, int ilo, int ihi, int cdone, int mode,
                           double *r, int64_t rinc, double *c, int64_t cinc, double *kappa,
                           const FtFix *fixes, int nfix, double *deltas, cudaStream_t s);
cudaError_t ft_frob_to_ctl(const double *A, int lda, int n, FtCtl *ctl, cudaStream_t s);
cudaError_t ft_build_v(const double *Aw, int64_t ldw, double *V, int n, int ihi, int k, int ib, cudaStream_t s,
                       const FtCtl *ctl = nullptr, int vchk = 0);
// gpart: Gram partial workspace of (ihi-k-1)/128 + 1 blocks of 64 x 64 doubles
cudaError_t ft_larft(const double *V, int64_t ldw, const double *tau, double *T, int n, int ihi, int k,
                     int ib, cudaStream_t s, const FtCtl *ctl, double *gpart);
cudaError_t ft_set_identity(double *Q, int64_t ldq, int n, cudaStream_t s);
cudaError_t ft_set_identity_aug(double *Q, int64_t ldq, int n, cudaStream_t s);
cudaError_t ft_ctl_set_norm(FtCtl *ctl, double v, cudaStream_t s);

#ifdef __cplusplus
#include <vector>
#include <mutex>
std::recursive_mutex &ft_api_mutex();  // held by every public entry point (ft_driver.cu)
// the host R12 decoder (ft_driver.cu), shared with the multi-rank path: 0 clean, 1 fixes, 2 refused
int ft_host_decode(int n, const double *Dr, const double *Dc, double sr, double sc, double tau,
                   std::vector<FtFix> *fixes);
#endif

extern int64_t g_ft_launches;
extern int64_t g_ft_wide_launches;  // launches of the two-reduction (wide) panel kernel

// Bit of the current device in a per-device "attribute set" mask: kernel attributes such as the
// dynamic shared-memory opt-in belong to a device context, so one-time setup is keyed by device.
inline unsigned ft_dev_bit() {
    int dev = 0;
    cudaGetDevice(&dev);
    return 1u << (dev & 31);
}
