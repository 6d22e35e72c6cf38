// ft_driver.cu -- host orchestrator and C ABI of libftgehrd (FT_DGEHRD, Alg. 3 P:216,
// re-designed all-GPU: panel, updates, checksums, verification and injector all run in
// this library's kernels; the host only enqueues them and, on a detected error, drives
// the recovery (reverse computation P:260/P:316, location P:272, correction P:278).
//
// Fault-free calls enqueue every iteration back to back with no host synchronization:
// each kernel first reads a device "halt" word, and a check kernel that detects an
// inconsistency raises it, turning every later kernel of the call into a no-op.  The
// host reads the control block once at the end; if it finds a halt it recovers the
// iteration that raised it and re-enqueues from there.
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <tuple>
#include <vector>

#include "ft_internal.h"

#include <mutex>
// Every public entry point holds this process-wide lock for the whole call: the workspace, the cached
// graphs and the counters are shared per device, so calls from several host threads are serialised
// here instead of racing (a call blocks until its stream has finished anyway).  Recursive: entry
// points call each other (ft_dsytrd -> run, ft_dgehrd_host -> run).
std::recursive_mutex &ft_api_mutex() {
    static std::recursive_mutex mu;
    return mu;
}

int64_t g_ft_launches = 0;
int64_t g_ft_wide_launches = 0;
extern "C" int64_t ft_debug_wide_launches(int reset) {
    const int64_t v = g_ft_wide_launches;
    if (reset) g_ft_wide_launches = 0;
    return v;
}
static int g_dbg_panel = -1;
static unsigned long long *g_dbg_buf = nullptr;
static int g_dbg_mode = 0;
extern "C" void ft_debug_ablate(int mode) { g_dbg_mode = mode; }
static int g_panel_path = 0;  // OR'ed into every panel launch's mode bits (8: explicit path, 64/128: smem modes 1/0)
extern "C" void ft_debug_panel_path(int bits) { g_panel_path = bits & (8 | 64 | 128); }
static int g_left_fold = 1;  // ABFT left update: checksum row/column folded (1) or as DMMA tiles (0)
extern "C" void ft_debug_left_fold(int on) { g_left_fold = on ? 1 : 0; }
static int g_right_fold = 1;  // ABFT right update: checksum row c as a GEMV of the last row split (1) or a tile row (0)
extern "C" void ft_debug_right_fold(int on) { g_right_fold = on ? 1 : 0; }
extern "C" void ft_debug_probe_panel(int panel, unsigned long long *dbuf) {
    g_dbg_panel = panel;
    g_dbg_buf = dbuf;
}
// Live device timing with CUDA events on the launching stream.  Categories 1..7 are the report's
// phases (ft_report.ms, opts.timing); 8..10 the kernel classes of the bench's roofline (panel
// kernel, right-update launch, left-update launch; ft_debug_time_kernels).
enum { TC_PANEL = 1, TC_RIGHT = 2, TC_LEFT = 3, TC_VERIFY = 4, TC_RECOVERY = 5, TC_COPY = 6, TC_ENCODE = 7,
       TK_PANEL = 8, TK_RIGHT = 9, TK_LEFT = 10, TC_N = 11 };
static bool g_time_kernels = false;
static double g_kms[3] = {0.0, 0.0, 0.0};
static int g_kn[3] = {0, 0, 0};
extern "C" void ft_debug_time_kernels(int on) {
    g_time_kernels = on != 0;
    if (on)
        for (int q = 0; q < 3; q++) {
            g_kms[q] = 0.0;
            g_kn[q] = 0;
        }
}
extern "C" double ft_debug_kernel_ms(int cls) { return cls >= 0 && cls < 3 ? g_kms[cls] : 0.0; }
extern "C" int ft_debug_kernel_launches(int cls) { return cls >= 0 && cls < 3 ? g_kn[cls] : 0; }
extern "C" void ft_debug_time_panels(int on) { ft_debug_time_kernels(on); }
extern "C" double ft_debug_panel_ms(void) { return g_kms[0]; }
extern "C" int ft_debug_panel_launches(void) { return g_kn[0]; }

namespace {

const double kEps = 2.220446049250313e-16;

#define CK(x)                                        \
    do {                                             \
        cudaError_t e_ = (x);                        \
        if (e_ != cudaSuccess) {                     \
            if (getenv("FT_DEBUG"))                  \
                fprintf(stderr, "ftgehrd: %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
            return FT_E_CUDA;                        \
        }                                            \
    } while (0)

// ---------------------------------------------------------------------------
// workspace (cached per device, grown on demand)
// ---------------------------------------------------------------------------
constexpr int kMaxWsplit = FT_WSPLIT_MAX;
// Y_top split partials: up to kYtopSplits x (n+1) rows (or 296 x 64 rows for small n) kept in ypart
constexpr int kYtopSplits = 16;
int64_t ytop_rows_cap(int n) { return std::max<int64_t>(296 * 64, (int64_t)kYtopSplits * (n + 1)); }

struct Work {
    int n_cap = -1;
    int64_t ldw = 0;
    double *Wt = nullptr;
    double *Aw = nullptr, *V = nullptr, *Y = nullptr, *Z = nullptr, *T = nullptr, *Wpart = nullptr, *bvec = nullptr,
           *acc = nullptr, *ckpt = nullptr, *ck_r = nullptr, *ck_c = nullptr, *ck_q = nullptr, *Fr = nullptr,
           *Qr = nullptr, *Qc = nullptr, *Dr = nullptr, *Dc = nullptr, *sums = nullptr, *ypart = nullptr,
           *rowpart = nullptr, *linepart = nullptr, *scratch = nullptr, *deltas = nullptr, *hA = nullptr, *htau = nullptr,
           *ck_w = nullptr, *Dr2 = nullptr, *Dc2 = nullptr, *wpart = nullptr, *dec_delta = nullptr,
           *dpart = nullptr;  // deterministic mode: per-CTA column-dot partials (PanelParams::dpart)
    int *dec_idx = nullptr;       // device decoder: compacted flagged rows / columns (2n)
    FtFix *dec_fix = nullptr;     // its fix plan (n + 8)
    FtDecOut *dec_out = nullptr;  // [pass 1, pass 2]
    unsigned *bar = nullptr;
    int *strip_done = nullptr;
    cudaStream_t cap_stream = nullptr;  // graph capture stream (library-owned)
    cudaStream_t copy_stream = nullptr; // host-buffer calls: D2H of finished columns beside the panels
    cudaEvent_t copy_ev = nullptr;
    FtCtl *ctl = nullptr;
    FtFix *fixes = nullptr;
    int nsm = 0;
    size_t bytes = 0;
    void release() {
        double **ps[] = {&Wt, &Aw, &V, &Y, &Z, &T, &Wpart, &bvec, &acc, &ckpt, &ck_r, &ck_c, &ck_q, &Fr, &Qr, &Qc, &Dr, &Dc,
                         &sums, &ypart, &rowpart, &linepart, &scratch, &deltas, &hA, &htau, &ck_w, &Dr2, &Dc2, &wpart,
                         &dpart};
        for (auto p : ps) {
            if (*p) cudaFree(*p);
            *p = nullptr;
        }
        if (bar) cudaFree(bar);
        if (dec_idx) cudaFree(dec_idx);
        if (dec_fix) cudaFree(dec_fix);
        if (dec_out) cudaFree(dec_out);
        if (dec_delta) cudaFree(dec_delta);
        dec_idx = nullptr;
        dec_fix = nullptr;
        dec_out = nullptr;
        dec_delta = nullptr;
        if (strip_done) cudaFree(strip_done);
        strip_done = nullptr;
        if (ctl) cudaFree(ctl);
        if (fixes) cudaFree(fixes);
        bar = nullptr;
        ctl = nullptr;
        fixes = nullptr;
        n_cap = -1;
        bytes = 0;
    }
};
std::map<int, Work> g_work;

// CUDA graphs of fault-free calls, keyed by device, shape, options and caller buffers
struct GraphKey {
    int dev, n, ilo, ihi, nb, abft, policy, weighted, det;
    double c_thr;
    const void *dA;
    int lda;
    const void *dtau;
    bool operator<(const GraphKey &o) const {
        return std::tie(dev, n, ilo, ihi, nb, abft, policy, weighted, det, c_thr, dA, lda, dtau) <
               std::tie(o.dev, o.n, o.ilo, o.ihi, o.nb, o.abft, o.policy, o.weighted, o.det, o.c_thr, o.dA, o.lda,
                        o.dtau);
    }
};
struct GraphEntry {
    cudaGraphExec_t exec = nullptr;
    int64_t launches = 0;
    bool failed = false;
};
std::map<GraphKey, GraphEntry> g_graphs;
void drop_graphs(int dev) {
    for (auto it = g_graphs.begin(); it != g_graphs.end();) {
        if (it->first.dev == dev) {
            if (it->second.exec) cudaGraphExecDestroy(it->second.exec);
            it = g_graphs.erase(it);
        } else {
            ++it;
        }
    }
}

template <class T>
cudaError_t dalloc(T **p, size_t count, size_t &acc) {
    acc += count * sizeof(T);
    return cudaMalloc((void **)p, std::max<size_t>(count, 1) * sizeof(T));
}

int get_work(int n, Work **out) {
    int dev = 0;
    CK(cudaGetDevice(&dev));
    Work &w = g_work[dev];
    if (w.n_cap >= n) {
        *out = &w;
        return 0;
    }
    drop_graphs(dev);  // captured graphs hold the old workspace pointers
    w.release();
    int64_t ldw = ((int64_t)n + 2 + 31) / 32 * 32;
    size_t N1 = (size_t)n + 1;
    size_t b = 0;
    cudaError_t e = cudaSuccess;
    auto A = [&](cudaError_t x) {
        if (x != cudaSuccess && e == cudaSuccess) e = x;
    };
    A(dalloc(&w.Aw, (size_t)ldw * (N1 + 1), b));
    A(dalloc(&w.V, (size_t)ldw * FT_NBMAX, b));
    A(dalloc(&w.Y, (size_t)ldw * FT_NBMAX, b));
    A(dalloc(&w.T, (size_t)FT_NBMAX * FT_NBMAX, b));
    A(dalloc(&w.Wpart, (size_t)kMaxWsplit * (N1 + 64) * FT_NBMAX, b));
    A(dalloc(&w.Wt, (N1 + 64) * FT_NBMAX, b));
    A(dalloc(&w.Z, (size_t)ldw * FT_NBMAX, b));
    A(dalloc(&w.bvec, (size_t)4 * ldw, b));
    A(dalloc(&w.acc, (size_t)FT_ACC_SETS * FT_ACC_SET_DOUBLES, b));
    A(dalloc(&w.dpart, (size_t)FT_ACC_SETS * FT_ACC_STRIDE * FT_DPMAX, b));
    A(dalloc(&w.ckpt, (size_t)ldw * FT_NBMAX, b));
    A(dalloc(&w.ck_r, (size_t)ldw, b));
    A(dalloc(&w.ck_c, N1, b));
    A(dalloc(&w.ck_q, 3 * (size_t)ldw, b));
    A(dalloc(&w.Fr, (size_t)ldw, b));
    A(dalloc(&w.Qr, (size_t)ldw, b));
    A(dalloc(&w.Qc, (size_t)ldw, b));
    A(dalloc(&w.Dr, (size_t)ldw, b));
    A(dalloc(&w.Dc, (size_t)ldw, b));
    A(dalloc(&w.sums, 8, b));
    A(dalloc(&w.ypart, (size_t)ytop_rows_cap(n) * FT_NBMAX, b));
    A(dalloc(&w.rowpart, (size_t)ytop_rows_cap(n), b));
    A(dalloc(&w.scratch, (size_t)64 * ((n + 255) / 256) + 8, b));
    // row-sum partials of the verification ([64][ldw]) / Gram partials of Q formation's DLARFT
    A(dalloc(&w.linepart, (size_t)std::max<int64_t>(64 * ldw, 4096 * ((int64_t)n / 64 + 2)), b));
    A(dalloc(&w.deltas, (size_t)FT_MAX_EVENTS, b));
    A(dalloc(&w.ck_w, (size_t)2 * (n + 2), b));  // weighted pair (NEXT-1): checkpoint, syndromes, partials
    A(dalloc(&w.Dr2, (size_t)ldw, b));
    A(dalloc(&w.Dc2, (size_t)ldw, b));
    A(dalloc(&w.wpart, (size_t)128 * (n / 256 + 2), b));
    A(dalloc(&w.dec_idx, (size_t)2 * n + 2, b));
    A(dalloc(&w.dec_fix, (size_t)n + 8, b));
    A(dalloc(&w.dec_out, 2, b));
    A(dalloc(&w.dec_delta, (size_t)n + 8, b));
    A(dalloc(&w.bar, 4, b));
    A(dalloc(&w.strip_done, (N1 + 63) / 64 + 2, b));
    A(dalloc(&w.ctl, 1, b));
    A(dalloc(&w.fixes, (size_t)FT_MAX_EVENTS, b));
    if (e != cudaSuccess) {
        w.release();
        cudaGetLastError();
        return e == cudaErrorMemoryAllocation ? FT_E_NOMEM : FT_E_CUDA;
    }
    CK(cudaMemset(w.strip_done, 0, ((N1 + 63) / 64 + 2) * sizeof(int)));  // self-resetting afterwards
    CK(cudaMemset(w.V, 0, (size_t)ldw * FT_NBMAX * sizeof(double)));
    CK(cudaMemset(w.Y, 0, (size_t)ldw * FT_NBMAX * sizeof(double)));
    int nsm = 0;
    CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
    w.nsm = nsm;
    w.ldw = ldw;
    w.n_cap = n;
    w.bytes = b;
    *out = &w;
    return 0;
}

// ---------------------------------------------------------------------------
// R12 decoder (host side).  Works on the syndromes computed by the GPU full-verify
// kernels; emits a list of fixes that the GPU applies with explicit sums.
// Safety property: never miscorrect -- refuse whenever two explanations exist.
// ---------------------------------------------------------------------------
struct Plan {
    int status = 0;  // 0 clean, 1 fixes planned, 2 uncorrectable
    std::vector<FtFix> fixes;
};

bool bad(double d, double tau) { return !(std::fabs(d) <= tau); }
bool same(double a, double b, double tol) {
    bool fa = std::isfinite(a), fb = std::isfinite(b);
    if (!fa || !fb) return !fa && !fb;
    return std::fabs(a - b) <= tol;
}

// members of S whose syndromes add up to `target` (|subset| <= 3), unique, or fail
bool explain(const std::vector<int> &S, const std::vector<double> &D, double target, double tauS, int n,
             std::vector<int> &out) {
    out.clear();
    if (same(target, 0.0, tauS)) return true;
    if (!std::isfinite(target)) {
        for (int i : S)
            if (!std::isfinite(D[i])) out.push_back(i);
        return !out.empty() && out.size() <= 3;
    }
    if (S.size() > 256) return false;
    int hits = 0;
    std::vector<int> best;
    const size_t m = S.size();
    auto tol_of = [&](double s) { return tauS + 2.0 * n * kEps * s; };
    for (size_t a = 0; a < m; a++) {
        double da = D[S[a]];
        if (same(da, target, tol_of(std::fabs(da)))) {
            hits++;
            best = {S[a]};
        }
        for (size_t b2 = a + 1; b2 < m; b2++) {
            double db = D[S[b2]];
            if (same(da + db, target, tol_of(std::fabs(da) + std::fabs(db)))) {
                hits++;
                best = {S[a], S[b2]};
            }
            for (size_t c2 = b2 + 1; c2 < m; c2++) {
                double dc = D[S[c2]];
                if (same(da + db + dc, target, tol_of(std::fabs(da) + std::fabs(db) + std::fabs(dc)))) {
                    hits++;
                    best = {S[a], S[b2], S[c2]};
                }
            }
        }
    }
    if (hits != 1) return false;
    out = best;
    return true;
}

Plan decode(int n, const std::vector<double> &Dr, const std::vector<double> &Dc, double sr, double sc,
            double tau) {
    Plan P;
    const double tauS = tau * std::sqrt((double)std::max(n, 1));
    std::vector<int> R, C;
    for (int i = 0; i < n; i++)
        if (bad(Dr[i], tau)) R.push_back(i);
    for (int j = 0; j < n; j++)
        if (bad(Dc[j], tau)) C.push_back(j);
    const bool sr0 = same(sr, 0.0, tauS), sc0 = same(sc, 0.0, tauS);
    if (R.empty() && C.empty() && sr0 && sc0) return P;
    P.status = 2;
    if (R.empty() && C.empty()) {
        // only the corner: both sums off by the same amount
        if (!sr0 && !sc0 && same(sr, sc, tauS)) {
            P.fixes.push_back({-1, -1, 4, 0});
            P.status = 1;
        }
        return P;
    }
    // ambiguous with "corner + data errors"
    if (!sr0 && !sc0 && same(sr, sc, tauS)) return P;
    std::vector<int> Rc, Cc;
    if (!explain(R, Dr, sr, tauS, n, Rc) || !explain(C, Dc, sc, tauS, n, Cc)) return P;
    std::vector<int> Rd, Cd;
    for (int i : R)
        if (std::find(Rc.begin(), Rc.end(), i) == Rc.end()) Rd.push_back(i);
    for (int j : C)
        if (std::find(Cc.begin(), Cc.end(), j) == Cc.end()) Cd.push_back(j);
    auto pair_tol = [&](double a, double b) { return 2.0 * tau + 2.0 * n * kEps * (std::fabs(a) + std::fabs(b)); };
    // a flagged line without a flagged partner is a checksum word whose syndrome hid inside
    // the sum tolerance (tau < |d| <= tau sqrt(n)): accept if the whole set explains s_r / s_c
    auto whole_set = [&](const std::vector<int> &S, const std::vector<double> &D, double target) {
        if (S.size() > 3) return false;
        double sum = 0.0, sa = 0.0;
        for (int x : S) {
            if (!(std::fabs(D[x]) <= tauS)) return false;  // large syndromes cannot hide: a cancelling pair
            sum += D[x];
            sa += std::fabs(D[x]);
        }
        return same(sum, target, tauS + 2.0 * n * kEps * sa);
    };
    if (!Rd.empty() && Cd.empty() && whole_set(R, Dr, sr)) {
        Rc = R;
        Rd.clear();
    }
    if (!Cd.empty() && Rd.empty() && whole_set(C, Dc, sc)) {
        Cc = C;
        Cd.clear();
    }
    if (Rd.empty() != Cd.empty()) return P;
    if (!Rd.empty()) {
        if (Rd.size() == 1 && Cd.size() == 1) {
            if (!same(Dr[Rd[0]], Dc[Cd[0]], pair_tol(Dr[Rd[0]], Dc[Cd[0]]))) return P;
            P.fixes.push_back({Rd[0], Cd[0], 0, 0});
        } else if (Rd.size() == 1 || Cd.size() == 1) {
            // one shared line holds all errors: fix each along the orthogonal line
            const bool shared_row = Rd.size() == 1;
            const std::vector<int> &many = shared_row ? Cd : Rd;
            const std::vector<double> &Dm = shared_row ? Dc : Dr;
            double one = shared_row ? Dr[Rd[0]] : Dc[Cd[0]];
            double s = 0.0, sa = 0.0;
            bool nonfin = false;
            for (int x : many) {
                s += Dm[x];
                sa += std::fabs(Dm[x]);
                nonfin |= !std::isfinite(Dm[x]);
            }
            if (nonfin) {
                if (std::isfinite(one)) return P;
            } else if (!same(s, one, 2.0 * tauS + 2.0 * n * kEps * (sa + std::fabs(one)))) {
                return P;
            }
            for (int x : many) {
                if (shared_row) P.fixes.push_back({Rd[0], x, 1, 0});  // column formula
                else P.fixes.push_back({x, Cd[0], 0, 0});             // row formula
            }
        } else if (Rd.size() == Cd.size()) {
            std::vector<int> match(Rd.size(), -1);
            for (size_t a = 0; a < Rd.size(); a++) {
                int cnt = 0;
                for (size_t b2 = 0; b2 < Cd.size(); b2++)
                    if (same(Dr[Rd[a]], Dc[Cd[b2]], pair_tol(Dr[Rd[a]], Dc[Cd[b2]]))) {
                        cnt++;
                        match[a] = (int)b2;
                    }
                if (cnt != 1) return P;
            }
            for (size_t b2 = 0; b2 < Cd.size(); b2++) {
                int cnt = 0;
                for (size_t a = 0; a < Rd.size(); a++)
                    if (same(Dr[Rd[a]], Dc[Cd[b2]], pair_tol(Dr[Rd[a]], Dc[Cd[b2]]))) cnt++;
                if (cnt != 1) return P;
            }
            for (size_t a = 0; a < Rd.size(); a++) P.fixes.push_back({Rd[a], Cd[match[a]], 0, 0});
        } else {
            return P;
        }
    }
    for (int i : Rc) P.fixes.push_back({i, -1, 2, 0});
    for (int j : Cc) P.fixes.push_back({-1, j, 3, 0});
    P.status = 1;
    return P;
}

}  // namespace

// the R12 decoder for other translation units (the multi-rank path, ft_mgpu.cu): status 0 clean,
// 1 fixes planned, 2 uncorrectable
int ft_host_decode(int n, const double *Dr, const double *Dc, double sr, double sc, double tau,
                   std::vector<FtFix> *fixes) {
    std::vector<double> r(Dr, Dr + n), c(Dc, Dc + n);
    Plan P = decode(n, r, c, sr, sc, tau);
    if (fixes) *fixes = P.fixes;
    return P.status;
}

namespace {

// ---------------------------------------------------------------------------
// one call's state
// ---------------------------------------------------------------------------
struct Call {
    int n, ilo, ihi, nb, abft, policy;
    int weighted = 0;  // NEXT-1: the weighted checksum pair rides as row / column n+1
    int det = 0;       // opts.deterministic: fixed-order column-dot sums in the panel kernels
    // NEXT-4 (ft_dsytrd): symmetric input given by its lower triangle; d, e of the tridiagonal out
    int sym = 0;
    double *sym_d = nullptr, *sym_e = nullptr;
    double c_thr;
    cudaStream_t s;
    Work *w;
    double *tau;  // device tau (n-1)
    std::vector<ft_fault> faults;
    std::vector<ft_event> events;
    int detected = 0, corrected = 0, rollbacks = 0, redos = 0, uncorrectable = 0;
    int npanels = 0;
    int last = 0;           // panels enqueued by this call (stop_after_panel)
    int defer_from = -1;    // the next panel launch evaluates the end check of this iteration
    // host-buffer call (ft_dgehrd_host): the input is copied straight into the working array and
    // every iteration's finished columns [k, e) are copied back on w->copy_stream while the
    // following panels run (they are never touched again, except by a recovery: re-copied)
    double *hA = nullptr;
    int64_t hlda = 0;
    // Y_top fused into the panel (small n: every panel launch is narrow): the rows above the
    // panel ride through the panel's GEMV and Y recurrence (DLAHRD's formulation), and the
    // M-part of the right update is the b0 of those rows (written by the panel)
    bool fused_ytop = false;
    // event spans (category, start, stop) when this call is timed (opts.timing or kernel timing)
    bool timing = false;
    std::vector<std::tuple<int, cudaEvent_t, cudaEvent_t>> spans;
    int rend() const { return abft ? n + 1 : ihi; }
    int cend() const { return abft ? n + 1 : n; }
    int pk(int t) const { return ilo - 1 + t * nb; }
    int pib(int t) const { return std::min(nb, ihi - 2 - pk(t)); }
    void ev(int kind, int panel, int64_t i, int64_t j, double d) {
        ft_event e;
        e.kind = kind;
        e.panel = panel;
        e.i = i;
        e.j = j;
        e.delta = d;
        events.push_back(e);
    }
};

// open a timed span of category cat on the call's stream (-1: the call is not timed)
int span_begin(Call &C, int cat) {
    if (!C.timing) return -1;
    cudaEvent_t a = nullptr, b = nullptr;
    if (cudaEventCreate(&a) != cudaSuccess || cudaEventCreate(&b) != cudaSuccess) return -1;
    cudaEventRecord(a, C.s);
    C.spans.emplace_back(cat, a, b);
    return (int)C.spans.size() - 1;
}
void span_end(Call &C, int idx) {
    if (idx >= 0) cudaEventRecord(std::get<2>(C.spans[idx]), C.s);
}
// after the stream has finished: per-category sums (ms) and counts, events released
void spans_collect(Call &C, double *ms, int *cnt) {
    for (int q = 0; q < TC_N; q++) {
        ms[q] = 0.0;
        cnt[q] = 0;
    }
    for (auto &sp : C.spans) {
        float t = 0.f;
        if (cudaEventElapsedTime(&t, std::get<1>(sp), std::get<2>(sp)) == cudaSuccess) {
            ms[std::get<0>(sp)] += t;
            cnt[std::get<0>(sp)]++;
        }
        cudaEventDestroy(std::get<1>(sp));
        cudaEventDestroy(std::get<2>(sp));
    }
    C.spans.clear();
}

double *site_addr(Call &C, const ft_fault &f) {
    Work &w = *C.w;
    const int64_t ldw = w.ldw;
    const int n = C.n;
    switch (f.site) {
    case FT_SITE_A:
        if (f.i < 0 || f.i >= n || f.j < 0 || f.j >= n) return nullptr;
        return w.Aw + f.i + f.j * ldw;
    case FT_SITE_R:
        if (!C.abft || f.i < 0 || f.i >= n) return nullptr;
        return w.Aw + f.i + (int64_t)n * ldw;
    case FT_SITE_C:
        if (!C.abft || f.j < 0 || f.j >= n) return nullptr;
        return w.Aw + n + f.j * ldw;
    case FT_SITE_K:
        if (!C.abft) return nullptr;
        return w.Aw + n + (int64_t)n * ldw;
    case FT_SITE_Y:
        if (f.i < 0 || f.i > n || f.j < 0 || f.j >= FT_NBMAX) return nullptr;
        return w.Y + f.i + f.j * ldw;
    case FT_SITE_V:
        if (f.i < 0 || f.i > n || f.j < 0 || f.j >= FT_NBMAX) return nullptr;
        return w.V + f.i + f.j * ldw;
    case FT_SITE_T:
        if (f.i < 0 || f.i >= FT_NBMAX || f.j < 0 || f.j >= FT_NBMAX) return nullptr;
        return w.T + f.i + f.j * FT_NBMAX;
    case FT_SITE_RW:
        if (!C.weighted || f.i < 0 || f.i >= n) return nullptr;
        return w.Aw + f.i + (int64_t)(n + 1) * ldw;
    case FT_SITE_CW:
        if (!C.weighted || f.j < 0 || f.j >= n) return nullptr;
        return w.Aw + n + 1 + f.j * ldw;
    }
    return nullptr;
}

void fill_report(Call &C, const ft_opts &o, const FtCtl &hf, float ms, const double *span_ms, ft_report &R);
bool q_has_fault_after(const Call &C, int panel) {
    for (size_t q = 0; q < C.faults.size() && q < FT_MAXFAULTS; q++)
        if (C.faults[q].phase == FT_PHASE_AFTER_UPDATE && C.faults[q].panel == panel) return true;
    return false;
}
bool has_fault(const Call &C, int panel, int phase) {
    for (size_t q = 0; q < C.faults.size() && q < FT_MAXFAULTS; q++)
        if (C.faults[q].phase == phase && (phase == FT_PHASE_AT_END || C.faults[q].panel == panel)) return true;
    return false;
}

int inject_at(Call &C, int panel, int phase) {
    for (size_t q = 0; q < C.faults.size() && q < FT_MAXFAULTS; q++) {
        const ft_fault &f = C.faults[q];
        if (f.phase != phase) continue;
        if (phase != FT_PHASE_AT_END && f.panel != panel) continue;
        double *a = site_addr(C, f);
        if (!a) continue;
        CK(ft_inject(a, (int)q, f.bit, C.w->ctl, C.s));
    }
    return 0;
}

// checkpoint copy kernels must respect the halt word, so they are kernels, not memcpys
__global__ void k_ckpt(double *Aw, int64_t ldw, int n, int rend, int k, int ib, double *ckpt, double *ck_r,
                       double *ck_c, double *ck_q, const double *Qr, const double *Qc, const double *Fr,
                       int restore, const FtCtl *ctl, int check_halt) {
    if (check_halt && ctl->halt) return;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t panel_elems = (int64_t)ldw * ib;
    for (int64_t x = tid; x < panel_elems; x += stride) {
        int64_t i = x % ldw, j = x / ldw;
        if (i >= rend) continue;
        double *a = Aw + i + (k + j) * ldw;
        if (restore) *a = ckpt[x];
        else ckpt[x] = *a;
    }
    for (int64_t i = tid; i <= n; i += stride) {
        double *r = Aw + i + (int64_t)n * ldw;  // column n (r, kappa)
        double *c = Aw + n + i * ldw;            // row n (c)
        if (restore) {
            *r = ck_r[i];
            *c = ck_c[i];
            ((double *)Qr)[i] = ck_q[i];
            ((double *)Qc)[i] = ck_q[ldw + i];
            ((double *)Fr)[i] = ck_q[2 * ldw + i];
        } else {
            ck_r[i] = *r;
            ck_c[i] = *c;
            ck_q[i] = Qr[i];
            ck_q[ldw + i] = Qc[i];
            ck_q[2 * ldw + i] = Fr[i];
        }
    }
}

int checkpoint(Call &C, int t, int restore) {
    Work &w = *C.w;
    int k = C.pk(t), ib = C.pib(t);
    int64_t total = std::max<int64_t>(w.ldw * ib, C.n + 1);
    int blocks = (int)std::min<int64_t>((total + 255) / 256, 4 * (int64_t)w.nsm);
    g_ft_launches++;
    k_ckpt<<<blocks, 256, 0, C.s>>>(w.Aw, w.ldw, C.n, C.rend(), k, ib, w.ckpt, w.ck_r, w.ck_c, w.ck_q, w.Qr, w.Qc,
                                    w.Fr, restore, w.ctl, restore ? 0 : 1);
    CK(cudaGetLastError());
    return 0;
}

int right_update(Call &C, int t, double sign, int do_w, bool precheck = false) {
    Work &w = *C.w;
    const int k = C.pk(t), ib = C.pib(t), e = k + ib;
    GemmRightParams g{};
    g.A = w.Aw;
    g.lda = w.ldw;
    g.ldw = w.ldw;
    g.Y = w.Y;
    g.V = w.V;
    g.K = ib;
    g.sign = sign;
    g.Wpart = w.Wpart;
    g.wsplit_stride = ((int64_t)C.n + 1 + 64) * FT_NBMAX;
    g.ctl = sign < 0 ? w.ctl : nullptr;
    // M-part: rows 0..k of the panel columns k+1..e-1 (DGEHRD's DTRMM + DAXPY), as one extra
    // strip of the trailing launch (done by the panel itself when Y_top is fused)
    g.has_m = (C.fused_ytop && sign < 0) ? 0 : 1;
    g.m_r_hi = k + 1;
    g.m_c_lo = k + 1;
    g.m_c_hi = e;
    // trailing block (+ checksum row/column), fused with W = V^T A_new and W' = T^T W
    g.do_right = 1;
    g.r_lo = 0;
    g.r_hi = C.rend() + C.weighted;  // + row n+1 (c_w) / column n+1 (r_w) of the weighted pair
    g.c_lo = e;
    g.c_hi = C.cend() + C.weighted;
    g.wr_lo = k + 1;
    g.wr_hi = C.ihi;
    g.do_w = do_w;
    g.fold_row = (C.abft && !C.weighted) ? g_right_fold : 0;  // row n (c) as a GEMV of the last row split
    g.nsplit = ft_gemm_splits(g.r_lo, g.r_hi - g.fold_row, g.c_lo, g.c_hi, w.nsm, g.has_m, do_w ? g.wr_lo : g.r_hi);
    if (do_w) {
        g.Wt = w.Wt;
        g.T = w.T;
        g.transT = 1;
        g.strip_done = w.strip_done;
    }
    g.tctl = (C.abft && sign < 0 && do_w) ? w.ctl : nullptr;  // T checksum where W' = T^T W is formed
    if (precheck) {  // fused pre-update check (R15), decided by every CTA before it touches A
        g.pre_ctl = w.ctl;
        g.pre_n = C.n;
        g.pre_panel = t;
    }
    CK(ft_launch_gemm_right(g, C.s));
    return 0;
}

int left_update(Call &C, int t, double sign, int nsplit, int endcheck = 0, bool pre_reset = false) {
    Work &w = *C.w;
    const int k = C.pk(t), ib = C.pib(t), e = k + ib;
    GemmLeftParams g{};
    g.A = w.Aw;
    g.lda = w.ldw;
    g.ldw = w.ldw;
    g.V = w.V;
    g.T = w.T;
    g.Wpart = w.Wpart;
    g.Wt = w.Wt;
    g.r_lo = k + 1;
    g.r_hi = C.rend() + C.weighted;
    g.c_lo = e;
    g.c_hi = C.cend() + C.weighted;
    g.K = ib;
    g.nsplit = nsplit;
    g.wsplit_stride = ((int64_t)C.n + 1 + 64) * FT_NBMAX;
    g.transT = 1;
    g.sign = sign;
    g.ctl = sign < 0 ? w.ctl : nullptr;
    g.wt_ready = 1;  // W' was formed by the right-update launch (and is kept for a rollback)
    g.endcheck = endcheck;
    g.panel = t;
    g.policy = C.policy;
    g.n = C.n;
    g.Fr = w.Fr;
    g.ectl = w.ctl;
    g.pre_reset = pre_reset ? w.ctl : nullptr;
    g.fold = C.abft ? g_left_fold : 0;
    g.tctl = (C.abft && sign < 0) ? w.ctl : nullptr;
    CK(ft_launch_gemm_left(g, C.s));
    return 0;
}

int trailing_nsplit(Call &C, int t) {
    const int e = C.pk(t) + C.pib(t);
    return ft_gemm_splits(0, C.rend() + C.weighted, e, C.cend() + C.weighted, C.w->nsm);
}

// panel-kernel sync state: barrier counters and accumulator sets must be zero when a
// sequence of panel launches starts (the kernels recycle them afterwards)
int reset_panel_state(Call &C) {
    Work &w = *C.w;
    CK(cudaMemsetAsync(w.bar, 0, 4 * sizeof(unsigned), C.s));
    CK(cudaMemsetAsync(w.acc, 0, (size_t)FT_ACC_SETS * FT_ACC_SET_DOUBLES * sizeof(double), C.s));
    return 0;
}

int enqueue_panel(Call &C, int t) {
    Work &w = *C.w;
    const int n = C.n, k = C.pk(t), ib = C.pib(t);
    const bool eager = C.abft && C.policy == FT_POLICY_EAGER;
    if (inject_at(C, t, FT_PHASE_BEFORE_PANEL)) return FT_E_CUDA;
    PanelParams p{};
    if (C.abft) {  // the panel kernel takes the diskless checkpoint in its prologue
        p.ckpt = w.ckpt;
        p.ck_r = w.ck_r;
        p.ck_c = w.ck_c;
        p.ck_q = w.ck_q;
        p.Fr = w.Fr;
    }
    p.A = w.Aw;
    p.ldw = w.ldw;
    p.V = w.V;
    p.Y = w.Y;
    p.T = w.T;
    p.tau = C.tau;
    p.bvec = w.bvec;
    p.Z = w.Z;
    p.acc = w.acc;
    p.dpart = C.det ? w.dpart : nullptr;
    p.bar = w.bar + (t & 1);
    p.bar_next = w.bar + ((t + 1) & 1);
    p.ctl = w.ctl;
    p.Qr = w.Qr;
    p.Qc = w.Qc;
    p.n = n;
    p.ihi = C.ihi;
    p.k = k;
    p.ib = ib;
    p.abft = C.abft;
    p.verify = eager ? 1 : 0;
    const bool fuse_pre = eager && !has_fault(C, t, FT_PHASE_AFTER_PANEL);
    p.precheck_sums = fuse_pre ? 1 : 0;
    if (C.defer_from == t - 1 && t > 0) {  // the end check of iteration t-1, at this launch's entry
        p.echeck = 1;
        p.echeck_panel = t - 1;
        p.echeck_policy = C.policy;
    }
    C.defer_from = -1;
    p.dbg = (t == g_dbg_panel) ? g_dbg_buf : nullptr;
    p.dbg_mode = ((t == g_dbg_panel) ? g_dbg_mode : 0) | g_panel_path;
    {
        static const int rot = getenv("FT_PANEL_ROT") ? atoi(getenv("FT_PANEL_ROT")) : 0;  // probe experiments
        p.dbg_mode |= rot << 16;
    }
    const int gr = ft_panel_group_rows();
    p.rbase = C.fused_ytop ? 0 : ((k + 1) / gr) * gr;
    p.ytop = C.fused_ytop ? 1 : 0;
    int rendp = (C.rend() + gr - 1) / gr * gr;
    p.ngroups = (rendp - p.rbase) / gr;
    if (C.weighted) CK(ft_ckpt_w(w.Aw, w.ldw, n, w.ck_w, 0, w.ctl, C.s));
    const int sp_panel = span_begin(C, TC_PANEL);
    const int sp_kpanel = span_begin(C, TK_PANEL);
    CK(ft_launch_panel(p, w.nsm, C.s));
    span_end(C, sp_kpanel);
    // Y_top = A(0:k+1, k+1:ihi) V T (+ area-1 row sums), unless the panel formed it
    YtopParams y{};
    y.A = w.Aw;
    y.ldw = w.ldw;
    y.V = w.V;
    y.T = w.T;
    y.Y = w.Y;
    y.ypart = w.ypart;
    y.rowpart = w.rowpart;
    y.Fr = w.Fr;
    y.ctl = w.ctl;
    y.n = n;
    y.ihi = C.ihi;
    y.k = k;
    y.ib = ib;
    y.abft = C.abft;
    y.verify = eager ? 1 : 0;
    y.decide = fuse_pre ? 1 : 0;
    y.panel = t;
    const int ytm = ft_ytop_rows_per_cta();
    int nm = (k + 1 + ytm - 1) / ytm;
    int nkt = (C.ihi - k - 1 + 31) / 32;
    // splits over the long inner dimension: about ytop_f CTAs per SM in total (4 warps each)
    static const int ytop_f = getenv("FT_YTOP_F") ? atoi(getenv("FT_YTOP_F")) : 12;  // measured: 2 -> 12 saves 42 ms at C3
    int ns = std::max(1, std::min({(ytop_f * w.nsm) / nm, nkt / 2, 64}));
    while ((int64_t)ns * (k + 1) > ytop_rows_cap(w.n_cap)) ns--;
    y.nsplit = std::max(ns, 1);
    if (!C.fused_ytop) CK(ft_launch_ytop(y, C.s));
    // weighted pair: rows n+1 of V and Y (w^T V, c_w V T), part of the panel's output
    if (C.weighted) CK(ft_wchk(w.Aw, w.V, w.Y, w.T, w.ldw, n, C.ihi, k, ib, w.wpart, w.ctl, C.s));
    span_end(C, sp_panel);
    if (inject_at(C, t, FT_PHASE_AFTER_PANEL)) return FT_E_CUDA;
    if (eager && !fuse_pre) {
        // a fault is scheduled after the panel: recompute the check sums after it
        const int sp = span_begin(C, TC_VERIFY);
        CK(cudaMemsetAsync(w.ctl->eY, 0, sizeof(double) * 2 * FT_NBMAX * FT_ESTR, C.s));
        CK(ft_precheck(w.Y, w.V, w.ldw, n, C.ihi, k, ib, w.ctl, C.s));
        CK(ft_decide(w.Y, w.V, w.T, w.ldw, n, k, ib, t, w.ctl, C.s));
        span_end(C, sp);
    }
    {
        const int sp = span_begin(C, TC_RIGHT), sk = span_begin(C, TK_RIGHT);
        if (right_update(C, t, -1.0, 1, fuse_pre)) return FT_E_CUDA;
        span_end(C, sk);
        span_end(C, sp);
    }
    if (inject_at(C, t, FT_PHASE_AFTER_RIGHT)) return FT_E_CUDA;
    // the weighted pair (NEXT-1) takes the separate end check, which also sums r_w and c_w
    const bool fuse_end = C.abft && !C.weighted && !has_fault(C, t, FT_PHASE_AFTER_UPDATE);
    // deferred to the next panel launch's entry (no last-CTA chain on this launch's tail) when one
    // follows in this sequence with nothing injected in between
    const bool defer_end = fuse_end && t + 1 < C.last && !has_fault(C, t + 1, FT_PHASE_BEFORE_PANEL);
    {
        const int sp = span_begin(C, TC_LEFT), sk = span_begin(C, TK_LEFT);
        if (left_update(C, t, -1.0, trailing_nsplit(C, t), fuse_end ? (defer_end ? 2 : 1) : 0, fuse_pre))
            return FT_E_CUDA;
        if (defer_end) C.defer_from = t;
        span_end(C, sk);
        span_end(C, sp);
    }
    // weighted pair: the panel columns are final now -- their c_w entries (row n+1, which no update
    // kernel writes for them) re-encoded before the end check compares sum c_w with w^T L e
    if (C.weighted) CK(ft_cw_panel(w.Aw, w.ldw, n, C.ilo, C.ihi, k, k + ib, w.ctl, C.s));
    if (inject_at(C, t, FT_PHASE_AFTER_UPDATE)) return FT_E_CUDA;
    if (C.abft && !fuse_end) {
        const int sp = span_begin(C, TC_VERIFY);
        CK(ft_endcheck(w.Aw, w.ldw, n, C.ihi, k, ib, t, C.policy, w.Fr, w.ctl, C.s, C.weighted));
        span_end(C, sp);
    }
    if (C.hA) {  // columns [k, e) are final: back to the host beside the next panels
        CK(cudaEventRecord(w.copy_ev, C.s));
        CK(cudaStreamWaitEvent(w.copy_stream, w.copy_ev, 0));
        CK(cudaMemcpy2DAsync(C.hA + (int64_t)k * C.hlda, (size_t)C.hlda * sizeof(double), w.Aw + (int64_t)k * w.ldw,
                             (size_t)w.ldw * sizeof(double), n * sizeof(double), ib, cudaMemcpyDeviceToHost,
                             w.copy_stream));
    }
    return 0;
}

// full verify + decode + correct + re-verify.  mode 0: H (cdone finished columns), 1: Q.
// Returns 0 ok (clean or corrected), FT_E_UNCORRECTABLE, or an error.
// ---------------------------------------------------------------------------
// Weighted pair (NEXT-1, w_i = i + 1): decoder v3 on the host (written apart from the oracle's).
// v2 first on the plain syndromes; if it corrects, weighted words that still disagree are refreshed;
// if it refuses, the weighted syndromes locate: D_cw(j) / D_c(j) = w_i names row i of column j's one
// error (and a row likewise), repaired along the line that holds no other error; checksum words
// whose orthogonal direction is clean are refreshed; the result is re-verified.
// ---------------------------------------------------------------------------
struct WSyn {
    std::vector<double> Dr, Dc, Drw, Dcw, rw, cw;
    double sumr = 0, sumc = 0, kap = 0, krw = 0, kcw = 0;
};

int fetch_wsyn(Call &C, int cdone, WSyn &S) {
    Work &w = *C.w;
    const int n = C.n;
    const int64_t ldw = w.ldw;
    double *M = w.Aw;
    S.Dr.resize(n);
    S.Dc.resize(n);
    S.Drw.resize(n);
    S.Dcw.resize(n);
    S.rw.resize(n);
    S.cw.resize(n);
    CK(ft_full_verify(M, ldw, n, C.ilo, C.ihi, cdone, 0, M + (int64_t)n * ldw, 1, M + n, ldw, nullptr, w.Dr, w.Dc,
                      w.sums, w.linepart, C.s));
    CK(cudaMemcpyAsync(S.Dr.data(), w.Dr, n * sizeof(double), cudaMemcpyDeviceToHost, C.s));
    CK(cudaMemcpyAsync(S.Dc.data(), w.Dc, n * sizeof(double), cudaMemcpyDeviceToHost, C.s));
    double sums[2];
    CK(cudaMemcpyAsync(sums, w.sums, 2 * sizeof(double), cudaMemcpyDeviceToHost, C.s));
    CK(ft_full_verify_w(M, ldw, n, C.ilo, C.ihi, cdone, M + (int64_t)(n + 1) * ldw, M + n + 1, ldw, w.Dr2, w.Dc2,
                        w.linepart, C.s));
    CK(cudaMemcpyAsync(S.Drw.data(), w.Dr2, n * sizeof(double), cudaMemcpyDeviceToHost, C.s));
    CK(cudaMemcpyAsync(S.Dcw.data(), w.Dc2, n * sizeof(double), cudaMemcpyDeviceToHost, C.s));
    CK(cudaMemcpyAsync(S.rw.data(), M + (int64_t)(n + 1) * ldw, n * sizeof(double), cudaMemcpyDeviceToHost, C.s));
    CK(cudaMemcpy2DAsync(S.cw.data(), sizeof(double), M + n + 1, ldw * sizeof(double), sizeof(double), n,
                         cudaMemcpyDeviceToHost, C.s));
    double corner[3];
    CK(cudaMemcpyAsync(&corner[0], M + n + (int64_t)n * ldw, sizeof(double), cudaMemcpyDeviceToHost, C.s));
    CK(cudaMemcpyAsync(&corner[1], M + n + (int64_t)(n + 1) * ldw, sizeof(double), cudaMemcpyDeviceToHost, C.s));
    CK(cudaMemcpyAsync(&corner[2], M + n + 1 + (int64_t)n * ldw, sizeof(double), cudaMemcpyDeviceToHost, C.s));
    CK(cudaStreamSynchronize(C.s));
    S.sumr = sums[0];
    S.sumc = sums[1];
    S.kap = corner[0];
    S.krw = corner[1];
    S.kcw = corner[2];
    return 0;
}

// fixes one launch at a time, in order (a later fix may read a word an earlier one repaired)
int apply_seq(Call &C, int panel, int cdone, const std::vector<FtFix> &fx) {
    Work &w = *C.w;
    const int n = C.n;
    const int64_t ldw = w.ldw;
    double *M = w.Aw;
    for (const FtFix &f : fx) {
        CK(cudaMemcpyAsync(w.fixes, &f, sizeof(FtFix), cudaMemcpyHostToDevice, C.s));
        CK(ft_apply_fixes(M, ldw, n, C.ilo, C.ihi, cdone, 0, M + (int64_t)n * ldw, 1, M + n, ldw,
                          M + n + (int64_t)n * ldw, w.fixes, 1, w.deltas, C.s));
        double d = 0.0;
        CK(cudaMemcpyAsync(&d, w.deltas, sizeof(double), cudaMemcpyDeviceToHost, C.s));
        CK(cudaStreamSynchronize(C.s));
        const int kind = f.kind <= 1 ? FT_EV_FIX_DATA : f.kind == 2 ? FT_EV_FIX_R : f.kind == 3 ? FT_EV_FIX_C
                         : f.kind == 4 ? FT_EV_FIX_K : f.kind == 5 ? FT_EV_FIX_RW : f.kind == 6 ? FT_EV_FIX_CW
                                                                                     : FT_EV_FIX_KW;
        C.ev(kind, panel, f.i, f.j, d);
    }
    return 0;
}

// the index named by a weighted / plain syndrome ratio (w_x = x + 1), or -1 when the ratio is not
// within 1/4 of an integer in [1, n] after its rounding error (t, tw: the two thresholds)
int named_index(double Dw, double D, double t, double tw, int n) {
    if (!std::isfinite(Dw) || !std::isfinite(D) || !(std::fabs(D) > t)) return -1;
    const double rho = Dw / D;
    const double err = (tw + (double)n * t) / std::fabs(D) + 4.0 * n * kEps * std::fabs(rho);
    if (!(err < 0.25)) return -1;
    const double k = std::nearbyint(rho);
    if (!(std::fabs(rho - k) <= err) || k < 1.0 || k > (double)n) return -1;
    return (int)k - 1;
}

int verify_and_correct_w(Call &C, int panel, int cdone, bool *found) {
    Work &w = *C.w;
    const int n = C.n;
    FtCtl hctl;
    CK(cudaMemcpyAsync(&hctl, w.ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost, C.s));
    CK(cudaStreamSynchronize(C.s));
    const double tau = C.c_thr * n * kEps * hctl.normF, tw = tau * n;
    const double tauS = tau * std::sqrt((double)std::max(n, 1)), twS = tw * std::sqrt((double)std::max(n, 1));
    auto flagged_w = [&](const WSyn &S, int *nr, int *nc) {
        int a = 0, b = 0;
        for (int i = 0; i < n; i++) a += bad(S.Dr[i], tau) || bad(S.Drw[i], tw);
        for (int j = 0; j < n; j++) b += bad(S.Dc[j], tau) || bad(S.Dcw[j], tw);
        if (nr) *nr = a;
        if (nc) *nc = b;
        return a + b;
    };
    auto sums_ok = [&](const WSyn &S) {
        double srw = 0.0, scw = 0.0;
        for (int i = 0; i < n; i++) srw += S.rw[i];
        for (int j = 0; j < n; j++) scw += S.cw[j];
        return same(S.sumr, S.kap, tauS) && same(S.sumc, S.kap, tauS) && same(srw, S.krw, twS) && same(scw, S.kcw, twS);
    };
    WSyn S;
    if (fetch_wsyn(C, cdone, S)) return FT_E_CUDA;
    *found = false;
    int nr = 0, nc = 0;
    if (flagged_w(S, &nr, &nc) == 0 && sums_ok(S)) return 0;
    *found = true;
    C.ev(FT_EV_DETECT, panel, nr, nc, 0.0);
    C.detected++;
    auto fail = [&]() {
        C.ev(FT_EV_UNCORRECTABLE, panel, -1, -1, 0.0);
        C.uncorrectable++;
        return FT_E_UNCORRECTABLE;
    };
    Plan P = decode(n, S.Dr, S.Dc, S.sumr - S.kap, S.sumc - S.kap, tau);
    if (P.status == 1) {
        if (apply_seq(C, panel, cdone, P.fixes)) return FT_E_CUDA;
        if (fetch_wsyn(C, cdone, S)) return FT_E_CUDA;
    }
    std::vector<FtFix> fx;
    if (P.status != 2) {
        // the data are verified: weighted words that still disagree are refreshed
        for (int i = 0; i < n; i++)
            if (bad(S.Drw[i], tw)) fx.push_back({i, -1, 5, 0});
        for (int j = 0; j < n; j++)
            if (bad(S.Dcw[j], tw)) fx.push_back({-1, j, 6, 0});
    } else {
        // weighted location, pass by pass (each pass can free lines for the next: L-shapes)
        for (int pass = 0; pass < 8; pass++) {
            int a = 0, b = 0;
            for (int i = 0; i < n; i++) a += bad(S.Dr[i], tau);
            for (int j = 0; j < n; j++) b += bad(S.Dc[j], tau);
            if (a == 0 || b == 0) break;
            std::vector<int> pi(n, -1);
            std::vector<FtFix> step;
            for (int j = 0; j < n; j++) {
                if (!bad(S.Dc[j], tau)) continue;
                const int i = named_index(S.Dcw[j], S.Dc[j], tau, tw, n);
                if (i >= 0 && (bad(S.Dr[i], tau) || bad(S.Drw[i], tw))) pi[j] = i;
            }
            for (int j = 0; j < n; j++) {
                const int i = pi[j];
                if (i < 0) continue;
                const int jr = named_index(S.Drw[i], S.Dr[i], tau, tw, n);
                step.push_back({i, j, jr == j ? 0 : 1, 0});  // alone in its row: row formula; else column
            }
            for (int i = 0; i < n; i++) {
                if (!bad(S.Dr[i], tau)) continue;
                const int j = named_index(S.Drw[i], S.Dr[i], tau, tw, n);
                if (j < 0 || !(bad(S.Dc[j], tau) || bad(S.Dcw[j], tw)) || pi[j] >= 0) continue;
                step.push_back({i, j, 0, 0});
            }
            if (step.empty()) break;
            if (apply_seq(C, panel, cdone, step)) return FT_E_CUDA;
            if (fetch_wsyn(C, cdone, S)) return FT_E_CUDA;
        }
        // checksum words: refreshed only when the orthogonal direction shows no flag anywhere
        int anyR = 0, anyC = 0;
        flagged_w(S, &anyR, &anyC);
        if (anyR && !anyC)
            for (int i = 0; i < n; i++) {
                if (bad(S.Dr[i], tau)) fx.push_back({i, -1, 2, 0});
                if (bad(S.Drw[i], tw)) fx.push_back({i, -1, 5, 0});
            }
        if (anyC && !anyR)
            for (int j = 0; j < n; j++) {
                if (bad(S.Dc[j], tau)) fx.push_back({-1, j, 3, 0});
                if (bad(S.Dcw[j], tw)) fx.push_back({-1, j, 6, 0});
            }
    }
    if (!fx.empty()) {
        if (apply_seq(C, panel, cdone, fx)) return FT_E_CUDA;
        if (fetch_wsyn(C, cdone, S)) return FT_E_CUDA;
    }
    // corners: kappa when both plain sums are off by the same amount; the weighted corners from the
    // (now verified) weighted vectors
    fx.clear();
    if (!same(S.sumr, S.kap, tauS) && same(S.sumr, S.sumc, tauS)) fx.push_back({-1, -1, 4, 0});
    {
        double srw = 0.0, scw = 0.0;
        for (int i = 0; i < n; i++) srw += S.rw[i];
        for (int j = 0; j < n; j++) scw += S.cw[j];
        if (flagged_w(S, nullptr, nullptr) == 0) {
            if (!same(srw, S.krw, twS)) fx.push_back({-1, -1, 7, 0});
            if (!same(scw, S.kcw, twS)) fx.push_back({-1, -1, 8, 0});
        }
    }
    if (!fx.empty()) {
        if (apply_seq(C, panel, cdone, fx)) return FT_E_CUDA;
        if (fetch_wsyn(C, cdone, S)) return FT_E_CUDA;
    }
    if (flagged_w(S, nullptr, nullptr) != 0 || !sums_ok(S)) return fail();
    C.corrected++;
    return 0;
}

// M: the augmented working array (the reduction's Aw, or ft_dorghr's augmented Q); mode 0 reads its
// checksum column n / row n / corner, mode 1 the Q checksums of the Householder vectors
int verify_and_correct_host(Call &C, int panel, int cdone, int mode, bool *found, double *M);

// full verify -> R12 decode -> explicit-sum fixes -> re-verify -> decode, all enqueued on the device
// (k_decode, k_fix_dev); the host reads the outcome and the fix list once, for the report
int verify_and_correct(Call &C, int panel, int cdone, int mode, bool *found, double *M = nullptr) {
    if (C.weighted && mode == 0 && (!M || M == C.w->Aw)) return verify_and_correct_w(C, panel, cdone, found);
    Work &w = *C.w;
    const int n = C.n;
    const int64_t ldw = w.ldw;
    if (!M) M = w.Aw;
    double *r = mode == 0 ? M + (int64_t)n * ldw : w.Qr;
    double *c = mode == 0 ? M + n : w.Qc;
    const int64_t cinc = mode == 0 ? ldw : 1;
    double *kap = mode == 0 ? M + n + (int64_t)n * ldw : w.Qc + n;
    const int cap = n + 8;
    for (int pass = 0; pass < 2; pass++) {
        CK(ft_full_verify(M, ldw, n, C.ilo, C.ihi, cdone, mode, r, 1, c, cinc, nullptr, w.Dr, w.Dc, w.sums,
                          w.linepart, C.s));
        CK(ft_decode(w.Dr, w.Dc, w.sums, kap, n, mode, w.ctl, w.dec_idx, w.dec_fix, cap, w.dec_out + pass, C.s));
        if (pass == 0)
            CK(ft_apply_fixes_dev(M, ldw, n, C.ilo, C.ihi, cdone, mode, r, 1, c, cinc, kap, w.dec_fix, cap,
                                  w.dec_delta, w.dec_out, C.s));
    }
    FtDecOut d[2];
    CK(cudaMemcpyAsync(d, w.dec_out, 2 * sizeof(FtDecOut), cudaMemcpyDeviceToHost, C.s));
    CK(cudaStreamSynchronize(C.s));
    *found = false;
    if (d[0].status == 0) return 0;
    if (d[0].status == 3) return verify_and_correct_host(C, panel, cdone, mode, found, M);  // (unreachable: cap)
    *found = true;
    C.ev(FT_EV_DETECT, panel, d[0].nR, d[0].nC, 0.0);
    C.detected++;
    if (d[0].status == 2) {
        C.ev(FT_EV_UNCORRECTABLE, panel, d[0].nR, d[0].nC, 0.0);
        C.uncorrectable++;
        return FT_E_UNCORRECTABLE;
    }
    const int nf = d[0].nfix;
    std::vector<FtFix> fx(nf);
    std::vector<double> dl(nf);
    CK(cudaMemcpy(fx.data(), w.dec_fix, nf * sizeof(FtFix), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(dl.data(), w.dec_delta, nf * sizeof(double), cudaMemcpyDeviceToHost));
    for (int q = 0; q < nf; q++) {
        const FtFix &f = fx[q];
        const int kind = f.kind == 0 || f.kind == 1 ? (mode == 0 ? FT_EV_FIX_DATA : FT_EV_FIX_Q)
                         : f.kind == 2             ? (mode == 0 ? FT_EV_FIX_R : FT_EV_FIX_QR)
                         : f.kind == 3             ? (mode == 0 ? FT_EV_FIX_C : FT_EV_FIX_QC)
                                                   : (mode == 0 ? FT_EV_FIX_K : FT_EV_FIX_QK);
        C.ev(kind, panel, f.i, f.j, dl[q]);
    }
    if (d[1].status != 0) {
        C.ev(FT_EV_UNCORRECTABLE, panel, -1, -1, 0.0);
        C.uncorrectable++;
        return FT_E_UNCORRECTABLE;
    }
    C.corrected++;
    return 0;
}

// the host copy of the same decision (R12), kept for a plan larger than the device's fix buffer
int verify_and_correct_host(Call &C, int panel, int cdone, int mode, bool *found, double *M) {
    Work &w = *C.w;
    const int n = C.n;
    const int64_t ldw = w.ldw;
    if (!M) M = w.Aw;
    double *r = mode == 0 ? M + (int64_t)n * ldw : w.Qr;
    int64_t rinc = 1;
    double *c = mode == 0 ? M + n : w.Qc;
    int64_t cinc = mode == 0 ? ldw : 1;
    double *kap = mode == 0 ? M + n + (int64_t)n * ldw : w.Qc + n;
    FtCtl hctl;
    CK(cudaMemcpyAsync(&hctl, w.ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost, C.s));
    CK(cudaStreamSynchronize(C.s));
    const double tau = mode == 0 ? C.c_thr * n * kEps * hctl.normF : C.c_thr * n * kEps * std::sqrt((double)n);
    std::vector<double> Dr(n), Dc(n);
    double sums[2], kh;
    *found = false;
    for (int pass = 0; pass < 2; pass++) {
        CK(ft_full_verify(M, ldw, n, C.ilo, C.ihi, cdone, mode, r, rinc, c, cinc, nullptr, w.Dr, w.Dc, w.sums,
                          w.linepart, C.s));
        CK(cudaMemcpyAsync(Dr.data(), w.Dr, n * sizeof(double), cudaMemcpyDeviceToHost, C.s));
        CK(cudaMemcpyAsync(Dc.data(), w.Dc, n * sizeof(double), cudaMemcpyDeviceToHost, C.s));
        CK(cudaMemcpyAsync(sums, w.sums, 2 * sizeof(double), cudaMemcpyDeviceToHost, C.s));
        CK(cudaMemcpyAsync(&kh, kap, sizeof(double), cudaMemcpyDeviceToHost, C.s));
        CK(cudaStreamSynchronize(C.s));
        Plan P = decode(n, Dr, Dc, sums[0] - kh, sums[1] - kh, tau);
        if (pass == 0) {
            // fault-free drift bookkeeping
            if (P.status == 0 || P.status == 1) {
                double mx = 0.0;
                for (int i = 0; i < n; i++) {
                    if (std::fabs(Dr[i]) <= tau) mx = std::max(mx, std::fabs(Dr[i]));
                    if (std::fabs(Dc[i]) <= tau) mx = std::max(mx, std::fabs(Dc[i]));
                }
                double unit = tau / C.c_thr;
                double rel = unit > 0 ? mx / unit : 0.0;
                unsigned long long bits;
                memcpy(&bits, &rel, 8);
                if (bits > hctl.drift_bits) {
                    CK(cudaMemcpyAsync(&w.ctl->drift_bits, &bits, 8, cudaMemcpyHostToDevice, C.s));
                }
            }
            if (P.status == 0) return 0;
            *found = true;
            int nr = 0, nc = 0;
            for (int i = 0; i < n; i++) {
                nr += bad(Dr[i], tau);
                nc += bad(Dc[i], tau);
            }
            C.ev(FT_EV_DETECT, panel, nr, nc, 0.0);
            C.detected++;
            if (P.status == 2) {
                C.ev(FT_EV_UNCORRECTABLE, panel, nr, nc, 0.0);
                C.uncorrectable++;
                return FT_E_UNCORRECTABLE;
            }
            // data fixes first, then the checksum refreshes (they read the repaired data); in chunks
            // of FT_MAX_EVENTS (a data error that propagated along its column before the final
            // verification of ft_dorghr is one fix per polluted row)
            const int nf = (int)P.fixes.size();
            std::vector<double> dl(nf);
            for (int q0 = 0; q0 < nf; q0 += FT_MAX_EVENTS) {
                const int m = std::min(FT_MAX_EVENTS, nf - q0);
                CK(cudaMemcpyAsync(w.fixes, P.fixes.data() + q0, m * sizeof(FtFix), cudaMemcpyHostToDevice, C.s));
                CK(ft_apply_fixes(M, ldw, n, C.ilo, C.ihi, cdone, mode, r, rinc, c, cinc, kap, w.fixes, m, w.deltas,
                                  C.s));
                CK(cudaMemcpyAsync(dl.data() + q0, w.deltas, m * sizeof(double), cudaMemcpyDeviceToHost, C.s));
                CK(cudaStreamSynchronize(C.s));
            }
            for (int q = 0; q < nf; q++) {
                const FtFix &f = P.fixes[q];
                int kind = f.kind == 0 || f.kind == 1 ? (mode == 0 ? FT_EV_FIX_DATA : FT_EV_FIX_Q)
                           : f.kind == 2             ? (mode == 0 ? FT_EV_FIX_R : FT_EV_FIX_QR)
                           : f.kind == 3             ? (mode == 0 ? FT_EV_FIX_C : FT_EV_FIX_QC)
                                                     : (mode == 0 ? FT_EV_FIX_K : FT_EV_FIX_QK);
                C.ev(kind, panel, f.i, f.j, dl[q]);
            }
        } else {
            if (P.status != 0) {
                C.ev(FT_EV_UNCORRECTABLE, panel, -1, -1, 0.0);
                C.uncorrectable++;
                return FT_E_UNCORRECTABLE;
            }
            C.corrected++;
        }
    }
    return 0;
}

int recover_body(Call &C, const FtCtl &h);
int recover(Call &C, const FtCtl &h) {
    const int sp = span_begin(C, TC_RECOVERY);
    const int rc = recover_body(C, h);
    span_end(C, sp);
    return rc;
}
int recover_body(Call &C, const FtCtl &h) {
    Work &w = *C.w;
    const int t = h.halt_panel;
    const int k = C.pk(t);
    // clear the halt so the recovery kernels run
    int zero = 0;
    CK(cudaMemcpyAsync(&w.ctl->halt, &zero, sizeof(int), cudaMemcpyHostToDevice, C.s));
    CK(cudaMemcpyAsync(&w.ctl->nflag, &zero, sizeof(int), cudaMemcpyHostToDevice, C.s));
    CK(cudaMemsetAsync(w.ctl->eY, 0, sizeof(double) * 2 * FT_NBMAX * FT_ESTR, C.s));
    CK(cudaMemsetAsync(w.ctl->sums, 0, sizeof(double) * 4, C.s));
    CK(cudaMemsetAsync(w.ctl->wsums, 0, sizeof(double) * 2, C.s));
    CK(cudaMemsetAsync(&w.ctl->done_count, 0, 3 * sizeof(int), C.s));  // done_count, done_ytop, done_left
    CK(cudaMemsetAsync(&w.ctl->tbad, 0, sizeof(int), C.s));
    if (h.halt_stage == 3) {
        // the right update ran with a T that failed its checksum (W' is void, the left update did not
        // run): undo the right update only, then redo the panel from its checkpoint
        if (right_update(C, t, +1.0, 0)) return FT_E_CUDA;
        C.ev(FT_EV_ROLLBACK, t, h.halt_reason, 0, 0.0);
        C.rollbacks++;
    } else if (h.halt_stage == 2) {
        // reverse computation: add back the left, then the right update
        if (left_update(C, t, +1.0, trailing_nsplit(C, t))) return FT_E_CUDA;
        if (right_update(C, t, +1.0, 0)) return FT_E_CUDA;
        C.ev(FT_EV_ROLLBACK, t, h.halt_reason, 0, 0.0);
        C.rollbacks++;
    } else {
        C.ev(FT_EV_PANEL_REDO, t, h.halt_reason, 0, 0.0);
        C.redos++;
    }
    // restore the pre-factorized panel and the checksum vectors (diskless checkpoint)
    if (checkpoint(C, t, 1)) return FT_E_CUDA;
    if (C.weighted) CK(ft_ckpt_w(w.Aw, w.ldw, C.n, w.ck_w, 1, w.ctl, C.s));
    if (reset_panel_state(C)) return FT_E_CUDA;
    bool found = false;
    int info = verify_and_correct(C, t, k, 0, &found);
    return info;
}

// start of a call: control block, working array (A, zero padding, checksum row/column,
// P:218-224), panel sync state, encode (Alg. 3 l.2), Q checksums
int enqueue_start(Call &C, const double *dA, int lda) {
    Work &w = *C.w;
    const int n = C.n;
    cudaStream_t s = C.s;
    if (n > 1) CK(cudaMemsetAsync(C.tau, 0, (n - 1) * sizeof(double), s));
    CK(ft_ctl_init(w.ctl, C.c_thr, s));
    const int sp_copy = span_begin(C, TC_COPY);
    CK(cudaMemsetAsync(w.Aw, 0, (size_t)w.ldw * (n + 1) * sizeof(double), s));
    CK(cudaMemsetAsync(w.V, 0, (size_t)w.ldw * FT_NBMAX * sizeof(double), s));
    CK(cudaMemsetAsync(w.Y, 0, (size_t)w.ldw * FT_NBMAX * sizeof(double), s));
    if (C.hA)
        CK(cudaMemcpy2DAsync(w.Aw, (size_t)w.ldw * sizeof(double), C.hA, (size_t)C.hlda * sizeof(double),
                             n * sizeof(double), n, cudaMemcpyHostToDevice, s));
    else
        CK(ft_copy_in(dA, lda, w.Aw, w.ldw, n, s));
    if (C.sym) CK(ft_mirror_lower(w.Aw, w.ldw, n, s));
    span_end(C, sp_copy);
    CK(cudaMemsetAsync(w.bvec, 0, (size_t)4 * w.ldw * sizeof(double), s));  // b(q >= ihi) must read 0
    if (reset_panel_state(C)) return FT_E_CUDA;
    if (C.abft) {
        const int sp_enc = span_begin(C, TC_ENCODE);
        CK(ft_encode(w.Aw, w.ldw, n, w.ctl, w.scratch, w.linepart, s));
        if (C.weighted) CK(ft_encode_w(w.Aw, w.ldw, n, w.linepart, s));
        CK(cudaMemsetAsync(w.Fr, 0, w.ldw * sizeof(double), s));
        if (C.ilo > 1) CK(ft_frozen_init(w.Aw, w.ldw, n, C.ilo - 1, w.Fr, s));
        CK(cudaMemsetAsync(w.Qr, 0, w.ldw * sizeof(double), s));
        CK(cudaMemsetAsync(w.Qc, 0, w.ldw * sizeof(double), s));
        span_end(C, sp_enc);
    }
    return 0;
}

// final verification of the finished H (a12) and of the Householder vectors, enqueued with
// the panels: syndromes and the flag / drift decision on the device (k_final_flags); the host decoder
// runs only if a flag is set
int enqueue_final(Call &C) {
    Work &w = *C.w;
    const int n = C.n;
    const int64_t ldw = w.ldw;
    const int cdone = std::max(C.ihi - 1, C.ilo - 1);
    const int sp = span_begin(C, TC_VERIFY);
    CK(ft_full_verify(w.Aw, ldw, n, C.ilo, C.ihi, cdone, 0, w.Aw + (int64_t)n * ldw, 1, w.Aw + n, ldw, nullptr, w.Dr,
                      w.Dc, w.sums, w.linepart, C.s));
    CK(ft_final_flags(w.Dr, w.Dc, w.sums, w.Aw + n + (int64_t)n * ldw, n, 0, w.ctl, C.s));
    CK(ft_full_verify(w.Aw, ldw, n, C.ilo, C.ihi, cdone, 1, w.Qr, 1, w.Qc, 1, nullptr, w.Dr, w.Dc, w.sums,
                      w.linepart, C.s));
    CK(ft_final_flags(w.Dr, w.Dc, w.sums, w.Qc + n, n, 1, w.ctl, C.s));
    span_end(C, sp);
    return 0;
}

int validate(int n, int ilo, int ihi, const void *A, int lda, const void *tau, const ft_opts *o) {
    if (n < 0) return -1;
    if (ilo < 1 || ilo > std::max(1, n)) return -2;
    if (ihi < std::min(ilo, n) || ihi > n) return -3;
    if (n > 0 && !A) return -4;
    if (lda < std::max(1, n)) return -5;
    if (n > 1 && !tau) return -6;
    if (o) {
        if (o->nb < 0 || o->nb > FT_NBMAX) return -7;
        if (o->abft != 0 && o->abft != 1) return -7;
        if (o->weighted != 0 && (o->weighted != 1 || o->abft != 1)) return -7;  // NEXT-1 needs ABFT
        if (o->policy != FT_POLICY_EAGER && o->policy != FT_POLICY_PAPER) return -7;
        if (o->c_thr < 0.0 || !(o->c_thr == o->c_thr)) return -7;
        if (o->nfaults < 0 || o->nfaults > FT_MAXFAULTS || (o->nfaults > 0 && !o->faults)) return -7;
        if (o->stop_after_panel < -1) return -7;
        if (o->timing != 0 && o->timing != 1) return -7;
        if (o->deterministic != 0 && o->deterministic != 1) return -7;
    }
    return 0;
}

int run(int n, int ilo, int ihi, double *dA, int lda, double *dtau, const ft_opts *opts, double *hA = nullptr,
        int hlda = 0, double *sym_d = nullptr, double *sym_e = nullptr) {
    ft_opts o;
    ft_opts_default(&o);
    if (opts) o = *opts;
    int info = validate(n, ilo, ihi, hA ? hA : dA, hA ? hlda : lda, dtau, &o);
    if (info) return info;
    cudaStream_t s = (cudaStream_t)o.stream;
    if (n == 0) return 0;
    Call C;
    C.n = n;
    C.ilo = ilo;
    C.ihi = ihi;
    C.nb = o.nb > 0 ? o.nb : (n < 4096 ? 32 : 64);
    C.abft = o.abft;
    C.weighted = o.abft ? o.weighted : 0;
    C.det = o.deterministic;
    C.policy = o.policy;
    C.c_thr = o.c_thr > 0 ? o.c_thr : 2.0;
    C.s = s;
    C.tau = dtau;
    C.timing = o.timing != 0 || g_time_kernels;
    C.sym = sym_d != nullptr;
    C.sym_d = sym_d;
    C.sym_e = sym_e;
    for (int q = 0; q < o.nfaults; q++) C.faults.push_back(o.faults[q]);
    int rc = get_work(n, &C.w);
    if (rc) return rc;
    Work &w = *C.w;
    // Y_top fused into the panel when every panel launch is narrow (<= 24 rows per CTA) and the
    // rows above the panel are cheap to stream per column (measured: faster at n = 1024 / 2048,
    // slower at n = 3200, where the GEMV's L2 traffic starts to dominate the column)
    const int pctas = ft_panel_cta_cap() > 0 ? std::min(ft_panel_cta_cap(), w.nsm) : w.nsm;
    C.fused_ytop = (n + 1 + 7) / 8 <= 3 * pctas && n <= 2560 && !getenv("FT_NO_FUSED_YTOP");
    if (hA && o.stop_after_panel < 0) {
        C.hA = hA;
        C.hlda = hlda;
        if (!w.copy_stream) CK(cudaStreamCreateWithFlags(&w.copy_stream, cudaStreamNonBlocking));
        if (!w.copy_ev) CK(cudaEventCreateWithFlags(&w.copy_ev, cudaEventDisableTiming));
    }
    cudaEvent_t ev0, ev1;
    CK(cudaEventCreate(&ev0));
    CK(cudaEventCreate(&ev1));
    CK(cudaEventRecord(ev0, s));
    C.npanels = 0;
    for (int k = ilo - 1; k < ihi - 2; k += C.nb) C.npanels++;
    const int last = (o.stop_after_panel >= 0) ? std::min(o.stop_after_panel + 1, C.npanels) : C.npanels;
    C.last = last;
    // Fault-free calls replay one CUDA graph of the whole launch sequence (start-up kernels and
    // every iteration), captured on the second call with the same shape and buffers; the halt
    // protocol is unchanged (a halted graph's remaining kernels are no-ops, recovery follows).
    const bool graphable = C.faults.empty() && o.stop_after_panel < 0 && g_dbg_panel < 0 && !C.timing && !C.sym &&
                           !g_panel_path && g_left_fold && g_right_fold &&
                           !getenv("FT_NO_GRAPH");
    bool launched = false;
    // the fault-free final verification's decision is taken on the device (not for the weighted pair,
    // whose final verification always runs the host decoder v3)
    const bool dev_final = C.abft && !C.weighted && o.stop_after_panel < 0;
    if (graphable) {
        int dev = 0;
        CK(cudaGetDevice(&dev));
        GraphKey key{dev, n, ilo, ihi, C.nb, C.abft, C.policy, C.weighted, C.det, C.c_thr, C.hA ? (const void *)C.hA : (const void *)dA,
                     C.hA ? (int)C.hlda : lda, (const void *)dtau};
        auto it = g_graphs.find(key);
        if (it != g_graphs.end() && it->second.exec) {
            CK(cudaGraphLaunch(it->second.exec, s));
            g_ft_launches += it->second.launches;
            launched = true;
        } else if (it != g_graphs.end() && !it->second.failed) {  // second call: capture
            // record on a library-owned stream (the caller's may be the legacy default stream,
            // which cannot capture); the graph is then launched on the caller's stream
            cudaGraph_t graph = nullptr;
            const int64_t l0 = g_ft_launches;
            if (!w.cap_stream) CK(cudaStreamCreateWithFlags(&w.cap_stream, cudaStreamNonBlocking));
            int rc2 = 1;
            cudaError_t ce = cudaStreamBeginCapture(w.cap_stream, cudaStreamCaptureModeThreadLocal);
            if (ce == cudaSuccess) {
                C.s = w.cap_stream;
                rc2 = enqueue_start(C, dA, lda);
                for (int t = 0; t < last && !rc2; t++) rc2 = enqueue_panel(C, t);
                if (!rc2 && dev_final) rc2 = enqueue_final(C);
                if (C.hA && !rc2) {  // join the copy stream back into the capture
                    if (cudaEventRecord(w.copy_ev, w.copy_stream) != cudaSuccess ||
                        cudaStreamWaitEvent(w.cap_stream, w.copy_ev, 0) != cudaSuccess)
                        rc2 = 1;
                }
                ce = cudaStreamEndCapture(w.cap_stream, &graph);
                C.s = s;
            }
            cudaGraphExec_t exec = nullptr;
            if (!rc2 && ce == cudaSuccess && graph && cudaGraphInstantiate(&exec, graph, 0) == cudaSuccess) {
                it->second.exec = exec;
                it->second.launches = g_ft_launches - l0;
                g_ft_launches = l0;
                CK(cudaGraphLaunch(exec, s));
                g_ft_launches += it->second.launches;
                launched = true;
            } else {
                g_ft_launches = l0;
                cudaGetLastError();
                it->second.failed = true;
            }
            if (graph) cudaGraphDestroy(graph);
        } else {
            g_graphs[key] = GraphEntry{};
        }
    }
    if (!launched) {
        rc = enqueue_start(C, dA, lda);
        if (rc) return rc;
    }
    int t0 = launched ? last : 0, attempts = 0;
    info = 0;
    FtCtl h;
    bool final_enqueued = launched && dev_final;  // the captured graph holds it
    while (true) {
        for (int t = t0; t < last; t++) {
            rc = enqueue_panel(C, t);
            if (rc) return rc;
        }
        if (o.stop_after_panel < 0 && !final_enqueued) {
            if (inject_at(C, -1, FT_PHASE_AT_END)) return FT_E_CUDA;
            if (dev_final && enqueue_final(C)) return FT_E_CUDA;
        }
        final_enqueued = false;
        CK(cudaMemcpyAsync(&h, w.ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (!h.halt) break;
        if (++attempts > 4 * (C.npanels + 1) + (int)C.faults.size() * 4) {
            C.ev(FT_EV_UNCORRECTABLE, h.halt_panel, -1, -1, 0.0);
            C.uncorrectable++;
            info = FT_E_UNCORRECTABLE;
            break;
        }
        C.defer_from = -1;  // recovery re-checks: the redo starts without a pending end check
        rc = recover(C, h);
        if (rc == FT_E_UNCORRECTABLE) {
            info = rc;
            break;
        }
        if (rc) return rc;
        t0 = h.halt_panel;
    }
    if (info == 0 && o.stop_after_panel < 0 && C.abft) {
        // final verification (a12): the host decoder only where the device flagged (or always
        // for the weighted pair)
        const bool doH = !dev_final || (h.fflag & 1), doQ = !dev_final || (h.fflag & 2);
        if (doH || doQ) {
            bool found = false;
            const int cdone = std::max(ihi - 1, ilo - 1);
            const int sp = span_begin(C, TC_VERIFY);
            int r1 = doH ? verify_and_correct(C, -1, cdone, 0, &found) : 0;
            if (r1 == 0 && doQ) r1 = verify_and_correct(C, -1, cdone, 1, &found);
            span_end(C, sp);
            if (r1 == FT_E_UNCORRECTABLE) info = r1;
            else if (r1) return r1;
        }
    }
    if (C.hA) {
        // join the column copies, then the columns no iteration finished ([0, ilo-1), the last
        // ones) -- or all of them if a recovery or the final verification touched the matrix
        CK(cudaEventRecord(w.copy_ev, w.copy_stream));
        CK(cudaStreamWaitEvent(s, w.copy_ev, 0));
        const bool touched = attempts > 0 || C.corrected > 0 || C.detected > 0;
        const int k0 = touched ? n : ilo - 1;
        const int e1 = touched ? 0 : (C.npanels > 0 ? C.pk(C.npanels - 1) + C.pib(C.npanels - 1) : 0);
        auto d2h = [&](int c0, int c1) -> cudaError_t {
            if (c1 <= c0) return cudaSuccess;
            return cudaMemcpy2DAsync(C.hA + (int64_t)c0 * C.hlda, (size_t)C.hlda * sizeof(double),
                                     w.Aw + (int64_t)c0 * w.ldw, (size_t)w.ldw * sizeof(double), n * sizeof(double),
                                     c1 - c0, cudaMemcpyDeviceToHost, s);
        };
        if (touched) {
            CK(d2h(0, n));
        } else {
            CK(d2h(0, std::min(k0, n)));
            CK(d2h(std::max(e1, k0), n));
        }
    } else {
        const int sp = span_begin(C, TC_COPY);
        if (C.sym) CK(ft_copy_out_lower(w.Aw, w.ldw, dA, lda, n, C.sym_d, C.sym_e, s));
        else CK(ft_copy_out(w.Aw, w.ldw, dA, lda, n, s));
        span_end(C, sp);
    }
    if (o.stop_after_panel >= 0 && o.dchk_out && C.abft) {
        CK(cudaMemcpyAsync(o.dchk_out, w.Aw + (int64_t)n * w.ldw, n * sizeof(double), cudaMemcpyDeviceToDevice, s));
        CK(cudaMemcpy2DAsync(o.dchk_out + n, sizeof(double), w.Aw + n, w.ldw * sizeof(double), sizeof(double), n,
                             cudaMemcpyDeviceToDevice, s));
        CK(cudaMemcpyAsync(o.dchk_out + 2 * n, w.Aw + n + (int64_t)n * w.ldw, sizeof(double),
                           cudaMemcpyDeviceToDevice, s));
        if (C.weighted) {  // [.. | r_w | c_w | e^T L w | w^T L e]
            CK(cudaMemcpyAsync(o.dchk_out + 2 * n + 1, w.Aw + (int64_t)(n + 1) * w.ldw, n * sizeof(double),
                               cudaMemcpyDeviceToDevice, s));
            CK(cudaMemcpy2DAsync(o.dchk_out + 3 * n + 1, sizeof(double), w.Aw + n + 1, w.ldw * sizeof(double),
                                 sizeof(double), n, cudaMemcpyDeviceToDevice, s));
            CK(cudaMemcpyAsync(o.dchk_out + 4 * n + 1, w.Aw + n + (int64_t)(n + 1) * w.ldw, sizeof(double),
                               cudaMemcpyDeviceToDevice, s));
            CK(cudaMemcpyAsync(o.dchk_out + 4 * n + 2, w.Aw + n + 1 + (int64_t)n * w.ldw, sizeof(double),
                               cudaMemcpyDeviceToDevice, s));
        }
    }
    CK(cudaEventRecord(ev1, s));
    FtCtl hf;
    CK(cudaMemcpyAsync(&hf, w.ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    float ms = 0.f;
    cudaEventElapsedTime(&ms, ev0, ev1);
    double span_ms[TC_N];
    int span_cnt[TC_N];
    spans_collect(C, span_ms, span_cnt);
    if (g_time_kernels)
        for (int q = 0; q < 3; q++) {
            g_kms[q] += span_ms[TK_PANEL + q];
            g_kn[q] += span_cnt[TK_PANEL + q];
        }
    cudaEventDestroy(ev0);
    cudaEventDestroy(ev1);
    if (o.report) fill_report(C, o, hf, ms, span_ms, *o.report);
    return info;
}

// the caller's report: injection events (fault order), then the detection / correction log
void fill_report(Call &C, const ft_opts &o, const FtCtl &hf, float ms, const double *span_ms, ft_report &R) {
    {
        memset(&R, 0, sizeof(R));
        // injection events first (in fault order), then the detection/correction log
        std::vector<ft_event> all;
        for (size_t q = 0; q < C.faults.size() && q < FT_MAXFAULTS; q++) {
            if (!hf.inj_done[q]) continue;
            ft_event e;
            e.kind = FT_EV_INJECT;
            e.panel = C.faults[q].phase == FT_PHASE_AT_END ? -1 : C.faults[q].panel;
            e.i = C.faults[q].i;
            e.j = C.faults[q].j;
            e.delta = hf.inj_delta[q];
            all.push_back(e);
        }
        all.insert(all.end(), C.events.begin(), C.events.end());
        R.nevents = (int)std::min<size_t>(all.size(), FT_MAX_EVENTS);
        for (int q = 0; q < R.nevents; q++) R.events[q] = all[q];
        R.detected = C.detected;
        R.corrected = C.corrected;
        R.rollbacks = C.rollbacks;
        R.panel_redos = C.redos;
        R.uncorrectable = C.uncorrectable;
        double drift;
        memcpy(&drift, &hf.drift_bits, 8);
        R.max_drift_rel = drift;
        R.ms[0] = ms;
        for (int q = 1; q < 8; q++) R.ms[q] = o.timing ? span_ms[q] : -1.0;
    }
}

// ---------------------------------------------------------------------------
// Q formation (DORGHR semantics; Q = H(ilo) ... H(ihi-1)), blocked and backward: for panel
// t = npanels-1 .. 0, Q(k+1:, k+1:) = (I - V T V^T) Q(k+1:, k+1:) (DLARFB 'L','N','F','C') as
// W = V^T Q (the right-update kernel's W pass) and Q -= V (T W) (the left-update kernel).
// With opts.abft = 1 (NEXT-3; P:266/P:278 protect Q's Householder vectors, this protects
// the accumulation): Q is carried augmented -- column n = r = Q e, row n = c = e^T Q, corner
// kappa = e^T Q e, encoded from Q = I -- and the same Theorem-1 algebra keeps them
// valid through every left update (V_chk = e^T V as row n of V; the left kernel folds r, c, kappa).
// Every iteration ends with the fused sum check (sum r = sum c = kappa; catches checksum-vector
// errors, rolled back with the retained W' and located); the end verifies Q against r, c and
// corrects with the R12 decoder.  A data error only ever mixes within its own column (left
// multiplications), so it is located at the end as one column with many rows, each repaired with
// the row formula.
// ---------------------------------------------------------------------------
double *q_scratch(int n, int64_t ldw, size_t cols, int *rc) {
    static std::map<int, std::pair<size_t, double *>> qscratch;
    int dev = 0;
    *rc = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) {
        *rc = FT_E_CUDA;
        return nullptr;
    }
    auto &qs = qscratch[dev];
    size_t need = (size_t)ldw * cols;
    if (qs.first < need) {
        if (qs.second) cudaFree(qs.second);
        qs.second = nullptr;
        qs.first = 0;
        if (cudaMalloc(&qs.second, need * sizeof(double)) != cudaSuccess) {
            cudaGetLastError();
            *rc = FT_E_NOMEM;
            return nullptr;
        }
        qs.first = need;
    }
    return qs.second;
}

int q_inject(Call &C, double *Qa, int panel, int phase) {
    const int64_t ldw = C.w->ldw;
    const int n = C.n;
    for (size_t q = 0; q < C.faults.size() && q < FT_MAXFAULTS; q++) {
        const ft_fault &f = C.faults[q];
        if (f.phase != phase || (phase != FT_PHASE_AT_END && f.panel != panel)) continue;
        double *a = nullptr;
        if (f.site == FT_SITE_A && f.i >= 0 && f.i < n && f.j >= 0 && f.j < n) a = Qa + f.i + f.j * ldw;
        else if (f.site == FT_SITE_R && f.i >= 0 && f.i < n) a = Qa + f.i + (int64_t)n * ldw;
        else if (f.site == FT_SITE_C && f.j >= 0 && f.j < n) a = Qa + n + f.j * ldw;
        else if (f.site == FT_SITE_K) a = Qa + n + (int64_t)n * ldw;
        if (a) CK(ft_inject(a, (int)q, f.bit, C.w->ctl, C.s));
    }
    return 0;
}

int dorghr_run(int n, int ilo, int ihi, const double *dA, int lda, const double *dtau, double *dQ, int ldq,
               const ft_opts &o) {
    cudaStream_t s = (cudaStream_t)o.stream;
    Call C;
    C.n = n;
    C.ilo = ilo;
    C.ihi = ihi;
    C.nb = o.nb > 0 ? o.nb : (n < 4096 ? 32 : 64);
    C.abft = o.abft;
    C.policy = FT_POLICY_EAGER;
    C.c_thr = o.c_thr > 0 ? o.c_thr : 2.0;
    C.s = s;
    C.timing = o.timing != 0;
    for (int q = 0; q < o.nfaults; q++) C.faults.push_back(o.faults[q]);
    int rc = get_work(n, &C.w);
    if (rc) return rc;
    Work &w = *C.w;
    const bool ab = C.abft != 0;
    cudaEvent_t ev0, ev1;
    CK(cudaEventCreate(&ev0));
    CK(cudaEventCreate(&ev1));
    CK(cudaEventRecord(ev0, s));
    CK(ft_ctl_init(w.ctl, C.c_thr, s));
    if (ab) CK(ft_ctl_set_norm(w.ctl, std::sqrt((double)n), s));  // ||Q||_F = sqrt(n) (R10 scale of Q)
    CK(ft_copy_in(dA, lda, w.Aw, w.ldw, n, s));  // private copy of V (dQ may alias dA)
    // the DMMA tiles move 16-byte chunks: work in an aligned scratch if dQ / ldq are not (and always
    // with ABFT: the augmented Q has a checksum row and column)
    double *Qw = dQ;
    int64_t ldqw = ldq;
    if (ab || (ldq & 1) || (((uintptr_t)dQ) & 15)) {
        Qw = q_scratch(n, w.ldw, (size_t)n + 1, &rc);
        if (rc) return rc;
        ldqw = w.ldw;
    }
    if (ab) CK(ft_set_identity_aug(Qw, ldqw, n, s));
    else CK(ft_set_identity(Qw, ldqw, n, s));
    int npanels = 0;
    for (int k = ilo - 1; k < ihi - 2; k += C.nb) npanels++;
    C.npanels = npanels;
    const int rend = ab ? n + 1 : ihi, cend = ab ? n + 1 : ihi;
    auto enqueue_q = [&](int t) -> int {
        const int k = ilo - 1 + t * C.nb, ib = std::min(C.nb, ihi - 2 - k);
        if (ab && q_inject(C, Qw, t, FT_PHASE_BEFORE_PANEL)) return FT_E_CUDA;
        CK(ft_build_v(w.Aw, w.ldw, w.V, n, ihi, k, ib, s, ab ? w.ctl : nullptr, ab ? 1 : 0));
        CK(ft_larft(w.V, w.ldw, dtau, w.T, n, ihi, k, ib, s, ab ? w.ctl : nullptr, w.linepart));
        GemmRightParams g{};
        g.A = Qw;
        g.lda = ldqw;
        g.ldw = w.ldw;
        g.Y = nullptr;
        g.V = w.V;
        g.r_lo = k + 1;
        g.r_hi = ihi;
        g.c_lo = k + 1;
        g.c_hi = cend;
        g.K = ib;
        g.wr_lo = k + 1;
        g.wr_hi = ihi;
        g.do_right = 0;
        g.do_w = 1;
        g.sign = 1.0;
        g.Wpart = w.Wpart;
        g.wsplit_stride = ((int64_t)n + 1 + 64) * FT_NBMAX;
        const int ns = ft_gemm_splits(k + 1, ihi, k + 1, cend, w.nsm);
        g.nsplit = ns;
        g.ctl = ab ? w.ctl : nullptr;
        g.Wt = w.Wt;
        g.T = w.T;
        g.transT = 0;
        g.strip_done = w.strip_done;
        {
            const int sp = span_begin(C, TC_RIGHT);
            CK(ft_launch_gemm_right(g, s));
            span_end(C, sp);
        }
        GemmLeftParams L{};
        L.A = Qw;
        L.lda = ldqw;
        L.ldw = w.ldw;
        L.V = w.V;
        L.T = w.T;
        L.Wpart = w.Wpart;
        L.Wt = w.Wt;
        L.r_lo = k + 1;
        L.r_hi = rend;
        L.c_lo = k + 1;
        L.c_hi = cend;
        L.K = ib;
        L.nsplit = ns;
        L.wsplit_stride = g.wsplit_stride;
        L.transT = 0;
        L.sign = -1.0;
        L.ctl = ab ? w.ctl : nullptr;
        L.wt_ready = 1;
        if (ab) {  // checksum row / column folded, fused end-of-iteration sum check (no frozen sums)
            L.fold = 1;
            L.endcheck = q_has_fault_after(C, t) ? 0 : 1;
            L.panel = t;
            L.policy = FT_POLICY_EAGER;
            L.n = n;
            L.Fr = nullptr;
            L.ectl = w.ctl;
        }
        {
            const int sp = span_begin(C, TC_LEFT);
            CK(ft_launch_gemm_left(L, s));
            span_end(C, sp);
        }
        if (ab) {
            if (q_inject(C, Qw, t, FT_PHASE_AFTER_UPDATE)) return FT_E_CUDA;
            if (!L.endcheck) CK(ft_endcheck(Qw, ldqw, n, ihi, k, ib, t, FT_POLICY_EAGER, nullptr, w.ctl, s));
        }
        return 0;
    };
    int t0 = npanels - 1, attempts = 0;
    int result = 0;
    while (true) {
        for (int t = t0; t >= 0; t--) {
            rc = enqueue_q(t);
            if (rc) return rc;
        }
        if (!ab) break;
        FtCtl h;
        CK(cudaMemcpyAsync(&h, w.ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (!h.halt) break;
        if (++attempts > 4 * (npanels + 1) + (int)C.faults.size() * 4) {
            C.ev(FT_EV_UNCORRECTABLE, h.halt_panel, -1, -1, 0.0);
            C.uncorrectable++;
            result = FT_E_UNCORRECTABLE;
            break;
        }
        // reverse computation of the halted iteration (its V, T, W' are still in the workspace:
        // every later launch was a no-op), then locate and correct, redo
        const int sp = span_begin(C, TC_RECOVERY);
        const int t = h.halt_panel, k = ilo - 1 + t * C.nb, ib = std::min(C.nb, ihi - 2 - k);
        int zero = 0;
        CK(cudaMemcpyAsync(&w.ctl->halt, &zero, sizeof(int), cudaMemcpyHostToDevice, s));
        CK(cudaMemsetAsync(w.ctl->sums, 0, sizeof(double) * 4, s));
        CK(cudaMemsetAsync(&w.ctl->done_count, 0, 3 * sizeof(int), s));
        GemmLeftParams L{};
        L.A = Qw;
        L.lda = ldqw;
        L.ldw = w.ldw;
        L.V = w.V;
        L.T = w.T;
        L.Wpart = w.Wpart;
        L.Wt = w.Wt;
        L.r_lo = k + 1;
        L.r_hi = rend;
        L.c_lo = k + 1;
        L.c_hi = cend;
        L.K = ib;
        L.nsplit = 1;
        L.wsplit_stride = ((int64_t)n + 1 + 64) * FT_NBMAX;
        L.transT = 0;
        L.sign = +1.0;
        L.wt_ready = 1;
        L.fold = 1;
        L.n = n;
        CK(ft_launch_gemm_left(L, s));
        C.ev(FT_EV_ROLLBACK, t, h.halt_reason, 0, 0.0);
        C.rollbacks++;
        bool found = false;
        const int r1 = verify_and_correct(C, t, ilo - 1, 0, &found, Qw);
        span_end(C, sp);
        if (r1 == FT_E_UNCORRECTABLE) {
            result = r1;
            break;
        }
        if (r1) return r1;
        t0 = t;
    }
    if (ab && result == 0) {
        if (q_inject(C, Qw, -1, FT_PHASE_AT_END)) return FT_E_CUDA;
        bool found = false;
        const int sp = span_begin(C, TC_VERIFY);
        const int r1 = verify_and_correct(C, -1, ilo - 1, 0, &found, Qw);  // final verification of Q
        span_end(C, sp);
        if (r1 == FT_E_UNCORRECTABLE) result = r1;
        else if (r1) return r1;
    }
    if (Qw != dQ) {
        const int sp = span_begin(C, TC_COPY);
        CK(cudaMemcpy2DAsync(dQ, (size_t)ldq * sizeof(double), Qw, (size_t)ldqw * sizeof(double),
                             (size_t)n * sizeof(double), n, cudaMemcpyDeviceToDevice, s));
        span_end(C, sp);
    }
    CK(cudaEventRecord(ev1, s));
    FtCtl hf;
    CK(cudaMemcpyAsync(&hf, w.ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    float ms = 0.f;
    cudaEventElapsedTime(&ms, ev0, ev1);
    cudaEventDestroy(ev0);
    cudaEventDestroy(ev1);
    double span_ms[TC_N];
    int span_cnt[TC_N];
    spans_collect(C, span_ms, span_cnt);
    if (o.report) fill_report(C, o, hf, ms, span_ms, *o.report);
    return result;
}

}  // namespace

// ---------------------------------------------------------------------------
// C ABI
// ---------------------------------------------------------------------------
extern "C" {

void ft_opts_default(ft_opts *o) {
    if (!o) return;
    memset(o, 0, sizeof(*o));
    o->nb = 0;
    o->abft = 1;
    o->weighted = 0;
    o->policy = FT_POLICY_EAGER;
    o->c_thr = 2.0;
    o->stop_after_panel = -1;
}

int ft_dgehrd(int n, int ilo, int ihi, double *dA, int lda, double *dtau, const ft_opts *opts) {
    std::lock_guard<std::recursive_mutex> api_lock(ft_api_mutex());
    return run(n, ilo, ihi, dA, lda, dtau, opts);
}

int ft_dsytrd(int n, double *dA, int lda, double *dd, double *de, double *dtau, const ft_opts *opts) {
    std::lock_guard<std::recursive_mutex> api_lock(ft_api_mutex());
    int info = validate(n, 1, n, dA, lda, dtau, nullptr);
    if (info) return info;
    if (n > 0 && !dd) return -4;
    if (n > 1 && !de) return -5;
    if (n == 0) return 0;
    if (n == 1) {  // no reflector: d = A(0,0)
        CK(cudaMemcpyAsync(dd, dA, sizeof(double), cudaMemcpyDeviceToDevice,
                           opts ? (cudaStream_t)opts->stream : (cudaStream_t)0));
        return 0;
    }
    return run(n, 1, n, dA, lda, dtau, opts, nullptr, 0, dd, de);
}

int ft_dgehrd_host(int n, int ilo, int ihi, double *hA, int lda, double *htau, const ft_opts *opts) {
    std::lock_guard<std::recursive_mutex> api_lock(ft_api_mutex());
    ft_opts o;
    ft_opts_default(&o);
    if (opts) o = *opts;
    int info = validate(n, ilo, ihi, hA, lda, htau, &o);
    if (info) return info;
    if (n == 0) return 0;
    cudaStream_t s = (cudaStream_t)o.stream;
    // device tau lives with the workspace of this size; A goes straight into the working array
    static std::map<int, std::pair<int, double *>> stage;
    int dev = 0;
    CK(cudaGetDevice(&dev));
    auto &st = stage[dev];
    if (st.first < n) {
        if (st.second) cudaFree(st.second);
        CK(cudaMalloc(&st.second, std::max(n, 2) * sizeof(double)));
        st.first = n;
    }
    double *dtau = st.second;
    if (o.stop_after_panel >= 0) {  // verify-hook calls: plain staging through a device copy
        double *dA = nullptr;
        CK(cudaMalloc(&dA, (size_t)n * n * sizeof(double)));
        CK(cudaMemcpy2DAsync(dA, n * sizeof(double), hA, (size_t)lda * sizeof(double), n * sizeof(double), n,
                             cudaMemcpyHostToDevice, s));
        info = run(n, ilo, ihi, dA, n, dtau, &o);
        if (!(info < 0 || info == FT_E_CUDA || info == FT_E_NOMEM))
            CK(cudaMemcpy2DAsync(hA, (size_t)lda * sizeof(double), dA, n * sizeof(double), n * sizeof(double), n,
                                 cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        cudaFree(dA);
    } else {
        info = run(n, ilo, ihi, nullptr, lda, dtau, &o, hA, lda);
    }
    if (info < 0 || info == FT_E_CUDA || info == FT_E_NOMEM) return info;
    if (n > 1) CK(cudaMemcpyAsync(htau, dtau, (n - 1) * sizeof(double), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    return info;
}

int ft_dorghr(int n, int ilo, int ihi, const double *dA, int lda, const double *dtau, double *dQ, int ldq,
              const ft_opts *opts) {
    std::lock_guard<std::recursive_mutex> api_lock(ft_api_mutex());
    ft_opts o;
    ft_opts_default(&o);
    if (opts) o = *opts;
    else o.abft = 0;  // NULL opts: the plain formation (documented)
    int info = validate(n, ilo, ihi, dA, lda, dtau, opts ? &o : nullptr);
    if (info) return info;
    if (n > 0 && !dQ) return -8;
    if (ldq < std::max(1, n)) return -9;
    if (o.nb < 0 || o.nb > FT_NBMAX) return -7;
    if (n == 0) return 0;
    return dorghr_run(n, ilo, ihi, dA, lda, dtau, dQ, ldq, o);
}

const char *ft_strerror(int info) {
    switch (info) {
    case 0: return "success";
    case FT_E_UNCORRECTABLE: return "uncorrectable soft error (checksum discrepancy could not be decoded)";
    case FT_E_CUDA: return "CUDA runtime error";
    case FT_E_NCCL: return "NCCL error";
    case FT_E_NOMEM: return "out of device memory";
    default: break;
    }
    if (info < 0) {
        static const char *args[] = {"", "n", "ilo", "ihi", "A", "lda", "tau", "opts", "Q / rank", "ldq / nranks"};
        static char buf[64];
        int a = -info;
        snprintf(buf, sizeof(buf), "illegal value of argument %d (%s)", a, a < 10 ? args[a] : "?");
        return buf;
    }
    return "unknown error";
}

void ft_finalize(void) {
    ft_mgpu_finalize();
    for (auto &kv : g_work) drop_graphs(kv.first);
    for (auto &kv : g_work) {
        int cur = 0;
        cudaGetDevice(&cur);
        cudaSetDevice(kv.first);
        kv.second.release();
        cudaSetDevice(cur);
    }
    g_work.clear();
}

const char *ft_version(void) { return "ftgehrd 0.1 (sm_100a; DMMA f64 updates, persistent DLAHR2 panel)"; }

int64_t ft_launch_count(int reset) {
    int64_t v = g_ft_launches;
    if (reset) g_ft_launches = 0;
    return v;
}

}  // extern "C"
