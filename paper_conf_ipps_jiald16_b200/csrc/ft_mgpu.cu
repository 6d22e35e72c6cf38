// ft_mgpu.cu -- multi-rank ABFT Hessenberg reduction: the n x n matrix is
// 1-D block-column cyclic over G ranks (block = nb); every rank holds all n rows of its
// columns plus a replicated row-checksum column r and the column checksums c of its own
// columns (row n).  Per panel (Alg. 3, on the sharded layout):
//   1. the owner of the panel block broadcasts its panel columns (rows 0..n) into every
//      rank's panel buffer P (peer stores over NVLink);
//   2. every rank runs the DLAHR2 panel redundantly on P; the trailing GEMV y = A(:, c+1:) v
//      (the hot spot) covers only the rank's own columns, and the per-column partials are
//      exchanged CTA by CTA inside the persistent panel kernel (ft_panel.cu, MG mode) -- no
//      collective on the host, one exchange per column, summed in rank order (identical on
//      every rank);
//   3. the owner copies P back; Y_top = A(0:k+1, k+1:n) V T is a per-rank partial over the
//      own columns, summed across ranks by a peer allreduce;
//   4. the right (+W) and left updates are rank-local on the own columns (+ the replicated r).
// Cross-rank kernels (exchange, panel) are "multi-rank launches": one launch covers every
// rank that lives on this GPU -- one per GPU in a real run (peers reached through CUDA IPC
// mappings of each rank's symmetric region), or G virtual ranks sharing one GPU (the test
// vehicle: identical kernels and protocol, peers are plain device pointers).
//
// Round-1 scope of the ABFT bookkeeping on this path: checksums (r, c, kappa) ride through
// every update exactly as on one GPU and the finished H is verified against them at the end
// (a12); detection is reported, correction/rollback run on the single-GPU path only.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "ft_common.cuh"
#include "ft_internal.h"

#include <mutex>

#define CK(x)                                                                                       \
    do {                                                                                            \
        cudaError_t e_ = (x);                                                                       \
        if (e_ != cudaSuccess) {                                                                    \
            if (getenv("FT_DEBUG")) fprintf(stderr, "ftgehrd: %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
            return FT_E_CUDA;                                                                       \
        }                                                                                           \
    } while (0)

namespace {

constexpr double kEpsM = 2.220446049250313e-16;

// ----------------------------------------------------------------------------------------
// generic cross-rank exchange (peer allreduce / broadcast of a 2-D region), multi-rank launch
// ----------------------------------------------------------------------------------------
struct XchgRank {
    double *src;                      // region base (column-major, leading dimension ld)
    int64_t ld;
    int rows, cols;
    int rank, G, mode, root;          // mode 0: allreduce (in place), 1: broadcast from root
    double *slot_peer[FT_MAX_VRANKS]; // every rank's exchange buffer for this parity [G][rows*cols]
    double *dst_peer[FT_MAX_VRANKS];  // broadcast: every rank's destination region base
    unsigned *fl_peer[FT_MAX_VRANKS]; // every rank's exchange flags [G][FT_FLAG_STRIDE]
    unsigned seq;
    const FtCtl *ctl;                 // halt-aware (every rank halts identically: its decision is taken
                                      // from allreduced values), or NULL
};
struct XchgLaunch {
    XchgRank r[FT_MAX_VRANKS];
    int nr;
};

__device__ __forceinline__ unsigned ld_acq_sys(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_rlx_sys(unsigned *p, unsigned v) {
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;\n" ::"l"(p), "r"(v) : "memory");
}

// block b of every rank handles the same element chunk; pairwise flags per (source, block)
__global__ void __launch_bounds__(256) k_xchg(const __grid_constant__ XchgLaunch L) {
    const int per = gridDim.x / L.nr;
    const int vr = blockIdx.x / per, bid = blockIdx.x % per;
    const XchgRank &x = L.r[vr];
    if (x.ctl && x.ctl->halt) return;
    const int64_t total = (int64_t)x.rows * x.cols;
    const int64_t e0 = total * bid / per, e1 = total * (bid + 1) / per;
    auto at = [&](double *base, int64_t e) -> double * { return base + (e % x.rows) + (e / x.rows) * x.ld; };
    if (x.mode == 0) {
        for (int64_t e = e0 + threadIdx.x; e < e1; e += blockDim.x) {
            const double v = *at(x.src, e);
            for (int g = 0; g < x.G; g++) x.slot_peer[g][(int64_t)x.rank * total + e] = v;
        }
    } else if (x.rank == x.root) {
        for (int64_t e = e0 + threadIdx.x; e < e1; e += blockDim.x) {
            const double v = *at(x.src, e);
            for (int g = 0; g < x.G; g++)
                if (g != x.root) *at(x.dst_peer[g], e) = v;
        }
    }
    __syncthreads();
    if (threadIdx.x == 0 && (x.mode == 0 || x.rank == x.root)) {
        __threadfence_system();
        for (int g = 0; g < x.G; g++) st_rlx_sys(x.fl_peer[g] + x.rank * FT_FLAG_STRIDE + bid, x.seq);
    }
    unsigned *own = x.fl_peer[x.rank];
    if (threadIdx.x < 32) {
        const int g = threadIdx.x;
        const bool need = g < x.G && (x.mode == 0 || g == x.root);
        if (need) {
            unsigned long long t0 = 0ull;
            unsigned polls = 0u;
            while (ld_acq_sys(own + g * FT_FLAG_STRIDE + bid) < x.seq) {
                peer_spin_guard(t0, polls);
            }
        }
    }
    __syncthreads();
    if (x.mode == 0) {
        const double *mine = x.slot_peer[x.rank];
        for (int64_t e = e0 + threadIdx.x; e < e1; e += blockDim.x) {
            double s = 0.0;
            for (int g = 0; g < x.G; g++) s += __ldcg(mine + (int64_t)g * total + e);  // rank order
            *at(x.src, e) = s;
        }
    }
}

// ----------------------------------------------------------------------------------------
// sharded-layout helpers
// ----------------------------------------------------------------------------------------
__global__ void k_mg_copy(const double *__restrict__ src, int64_t lds, double *__restrict__ dst, int64_t ldd, int rows,
                          int cols, const FtCtl *ctl) {
    if (ctl && ctl->halt) return;
    for (int64_t j = blockIdx.y; j < cols; j += gridDim.y)
        for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < rows; i += gridDim.x * blockDim.x)
            dst[i + j * ldd] = src[i + j * lds];
}
cudaError_t mg_copy(const double *src, int64_t lds, double *dst, int64_t ldd, int rows, int cols, cudaStream_t s,
                    const FtCtl *ctl = nullptr) {
    if (rows <= 0 || cols <= 0) return cudaSuccess;
    g_ft_launches++;
    k_mg_copy<<<dim3(std::min((rows + 255) / 256, 8), std::min(cols, 65535)), 256, 0, s>>>(src, lds, dst, ldd, rows,
                                                                                            cols, ctl);
    return cudaGetLastError();
}

// ----------------------------------------------------------------------------------------
// resilience on the sharded layout (round 2): checkpoint, end-of-iteration check on allreduced
// sums, reverse computation, distributed location and correction on the owners
// ----------------------------------------------------------------------------------------
// diskless checkpoint per rank: r and kappa (column ncl, rows 0..n), the own c
// entries (row n of the local columns), and on the owner the panel columns (rows 0..n)
__global__ void k_mg_ckpt(double *Aw, int64_t ldw, int n, int ncl, int lk, int ib, int owner, double *ck,
                          int restore, const FtCtl *ctl) {
    if (!restore && ctl->halt) return;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, st = (int64_t)gridDim.x * blockDim.x;
    double *rcol = Aw + (int64_t)ncl * ldw;
    for (int64_t i = tid; i <= n; i += st) {
        if (restore) rcol[i] = ck[i];
        else ck[i] = rcol[i];
    }
    double *cc = ck + n + 1;
    for (int64_t l = tid; l < ncl; l += st) {
        double *a = Aw + n + l * ldw;
        if (restore) *a = cc[l];
        else cc[l] = *a;
    }
    if (!owner) return;
    double *pp = cc + ncl;
    for (int64_t x = tid; x < (int64_t)(n + 1) * ib; x += st) {
        const int64_t i = x % (n + 1), j = x / (n + 1);
        double *a = Aw + i + (lk + j) * ldw;
        if (restore) *a = pp[x];
        else pp[x] = *a;
    }
}
// end-of-iteration sums: [sum r (rank 0's copy), sum of the own c entries, kappa (rank 0)]
__global__ void k_mg_endsums(const double *Aw, int64_t ldw, int n, int ncl, int rank, double *out, const FtCtl *ctl) {
    if (ctl->halt) return;
    __shared__ double red[2][32];
    double a = 0.0, b = 0.0;
    if (rank == 0)
        for (int i = threadIdx.x; i < n; i += blockDim.x) a += Aw[i + (int64_t)ncl * ldw];
    for (int l = threadIdx.x; l < ncl; l += blockDim.x) b += Aw[n + (int64_t)l * ldw];
    a = warp_sum(a);
    b = warp_sum(b);
    if ((threadIdx.x & 31) == 0) {
        red[0][threadIdx.x >> 5] = a;
        red[1][threadIdx.x >> 5] = b;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double x = 0.0, y = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
            x += red[0][w];
            y += red[1][w];
        }
        out[0] = x;
        out[1] = y;
        out[2] = rank == 0 ? Aw[n + (int64_t)ncl * ldw] : 0.0;
    }
}
// the decision (identical on every rank: it reads the rank-ordered allreduce of the sums): the paper's
// |sum r - sum c| and both sums against kappa (R22)
__global__ void k_mg_decide(const double *sums, int n, int panel, FtCtl *ctl) {
    if (ctl->halt) return;
    const double unit = (double)n * 2.220446049250313e-16 * ctl->normF;
    const double tauS = ctl->c_thr * unit * sqrt((double)n);
    const double Sr = sums[0], Sc = sums[1], kap = sums[2];
    if (not_within(Sr - Sc, tauS) || not_within(Sr - kap, tauS) || not_within(Sc - kap, tauS)) {
        ctl->halt_panel = panel;
        ctl->halt_stage = 2;
        ctl->halt_reason = 8;
        __threadfence();
        ctl->halt = 1;
    }
}
// the own columns' column discrepancies scattered into a full-length vector (others 0) for the
// allreduce, plus [sum r (rank 0), sum c (own), kappa (rank 0)] behind it
__global__ void k_mg_scatter_dc(const double *dc, int ncl, int G, int rank, int nb, int n, double *full) {
    for (int l = blockIdx.x * blockDim.x + threadIdx.x; l < ncl; l += gridDim.x * blockDim.x)
        full[ft_cmap(l, G, rank, nb, ncl, n)] = dc[l];
}
// apply located fixes: ops (row, local column, kind) with values; kind 0 add to A(i, l), 1 set r(i)
// (the replicated column), 2 add to c(l), 3 set kappa
struct MgOp {
    int64_t i, l;
    int kind, pad;
    double v;
};
__global__ void k_mg_apply(double *Aw, int64_t ldw, int n, int ncl, const MgOp *ops, int nops) {
    for (int q = blockIdx.x * blockDim.x + threadIdx.x; q < nops; q += gridDim.x * blockDim.x) {
        const MgOp o = ops[q];
        if (o.kind == 0) Aw[o.i + o.l * ldw] += o.v;
        else if (o.kind == 1) Aw[o.i + (int64_t)ncl * ldw] = o.v;
        else if (o.kind == 2) Aw[n + o.l * ldw] += o.v;
        else Aw[n + (int64_t)ncl * ldw] = o.v;
    }
}

// encode on the sharded layout: c(l) = column sums of the own columns (row n), partial row
// sums of the own columns into r (column ncl), ||A_local||_F^2 into scratch[0]
__global__ void k_mg_encode_cols(double *Aw, int64_t ldw, int n, int ncl, double *frob_part) {
    __shared__ double red[2][8];
    const int l = blockIdx.x;
    const double *col = Aw + (int64_t)l * ldw;
    double s = 0.0, q = 0.0;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
        const double a = col[i];
        s += a;
        q += a * a;
    }
    s = warp_sum(s);
    q = warp_sum(q);
    if ((threadIdx.x & 31) == 0) {
        red[0][threadIdx.x >> 5] = s;
        red[1][threadIdx.x >> 5] = q;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double ss = 0.0, qq = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
            ss += red[0][w];
            qq += red[1][w];
        }
        Aw[n + (int64_t)l * ldw] = ss;
        frob_part[l] = qq;
    }
}
// row sums of the own columns: r_part(i) = sum_l A(i, l)  (8 loads in flight per thread)
__global__ void k_mg_rowsums(const double *Aw, int64_t ldw, int n, int ncl, double *rpart) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        rpart[i] = ncl > 0 ? sum_strided(Aw + i, ldw, ncl) : 0.0;
}
// frobenius partial (sum over the per-column partials) into rpart[n]
__global__ void k_mg_frob(const double *frob_part, int ncl, double *out) {
    if (threadIdx.x == 0 && blockIdx.x == 0) *out = ncl > 0 ? sum_strided(frob_part, 1, ncl) : 0.0;
}
// after the allreduce: r column = summed row sums, kappa = sum r, normF into the control block
__global__ void k_mg_encode_finish(double *Aw, int64_t ldw, int n, int ncl, const double *rsum, FtCtl *ctl) {
    __shared__ double red[32];
    double s = 0.0;
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
        Aw[i + (int64_t)ncl * ldw] = rsum[i];
        s += rsum[i];
    }
    s = warp_sum(s);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double k = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); w++) k += red[w];
        Aw[n + (int64_t)ncl * ldw] = k;  // kappa = e^T A e
        ctl->normF = sqrt(rsum[n]);
    }
}

// final verification (a12) on the sharded layout: partial row sums of the logical H over the
// own columns (entries below the first subdiagonal hold Householder vectors: read as 0) and
// the own column discrepancies D_c(l) = c(l) - sum_i L(i, l)
__global__ void k_mg_verify_local(const double *Aw, int64_t ldw, int n, int ncl, int G, int rank, int nb,
                                  double *rpart, double *dc, int cdone) {
    // columns J < cdone are finished (logical H: rows 0..J+1; the stored Householder vectors read as
    // 0), the others are full columns of the working matrix
    const int tid = blockIdx.x * blockDim.x + threadIdx.x, stride = gridDim.x * blockDim.x;
    for (int i = tid; i < n; i += stride) {
        double s0 = 0.0, s1 = 0.0;
        for (int l = 0; l < ncl; l++) {
            const int J = ft_cmap(l, G, rank, nb, ncl, n);
            if (J >= cdone || i <= J + 1) {
                if (l & 1) s1 += Aw[i + (int64_t)l * ldw];
                else s0 += Aw[i + (int64_t)l * ldw];
            }
        }
        rpart[i] = s0 + s1;
    }
    for (int l = tid; l < ncl; l += stride) {
        const int J = ft_cmap(l, G, rank, nb, ncl, n);
        const int hi = J >= cdone ? n : std::min(J + 2, n);
        const double s = hi > 0 ? sum_strided(Aw + (int64_t)l * ldw, 1, hi) : 0.0;
        dc[l] = Aw[n + (int64_t)l * ldw] - s;
    }
}

// ----------------------------------------------------------------------------------------
// per-rank state
// ----------------------------------------------------------------------------------------
struct SymLayout {
    size_t P, yx, xbuf, flags, xflags, total;
    int64_t xlen;
};
SymLayout sym_layout(int64_t ldw, int G) {
    SymLayout L;
    size_t off = 0;
    auto take = [&](size_t bytes) {
        size_t o = off;
        off += (bytes + 255) / 256 * 256;
        return o;
    };
    L.xlen = ldw * FT_NBMAX;
    L.P = take((size_t)ldw * FT_NBMAX * sizeof(double));
    L.yx = take((size_t)2 * G * ldw * sizeof(double2));
    L.xbuf = take((size_t)2 * G * L.xlen * sizeof(double));
    L.flags = take((size_t)G * FT_FLAG_STRIDE * sizeof(unsigned));
    L.xflags = take((size_t)G * FT_FLAG_STRIDE * sizeof(unsigned));
    L.total = off;
    return L;
}

struct MgRank {
    int dev = -1, n_cap = -1, G = 0, rank = 0;
    int64_t ldw = 0;
    double *Aw = nullptr, *V = nullptr, *Y = nullptr, *Z = nullptr, *T = nullptr, *Wpart = nullptr, *Wt = nullptr, *bvec = nullptr,
           *acc = nullptr, *Qr = nullptr, *Qc = nullptr, *ypart = nullptr, *rowpart = nullptr, *vec = nullptr,
           *vec2 = nullptr, *ck = nullptr, *full = nullptr,
           *dpart = nullptr;  // deterministic mode: per-CTA column-dot partials (PanelParams::dpart)
    void *ops = nullptr;  // MgOp list of a correction
    unsigned *bar = nullptr;
    int *strip_done = nullptr;
    FtCtl *ctl = nullptr;
    char *sym = nullptr;  // symmetric region (own allocation)
    bool sym_owned = true;
    SymLayout lay{};
    char *peer[FT_MAX_VRANKS] = {};
    bool peer_opened[FT_MAX_VRANKS] = {};
    unsigned xseq = 0;  // generic exchange sequence (advanced identically on every rank)
    unsigned pseq = 0;  // panel flag base (advanced by n per call on every rank)
    int nsm = 0;
    double *P() const { return reinterpret_cast<double *>(sym + lay.P); }
    double2 *yx(int g) const { return reinterpret_cast<double2 *>(peer[g] + lay.yx); }
    double *xbuf(int g, int parity) const {
        return reinterpret_cast<double *>(peer[g] + lay.xbuf) + (int64_t)parity * G * lay.xlen;
    }
    unsigned *flags(int g) const { return reinterpret_cast<unsigned *>(peer[g] + lay.flags); }
    unsigned *xflags(int g) const { return reinterpret_cast<unsigned *>(peer[g] + lay.xflags); }
    void release() {
        double **ps[] = {&Aw, &V, &Y, &Z, &T, &Wpart, &Wt, &bvec, &acc, &Qr, &Qc, &ypart, &rowpart, &vec, &vec2, &ck, &full,
                         &dpart};
        for (auto p : ps) {
            if (*p) cudaFree(*p);
            *p = nullptr;
        }
        if (ops) cudaFree(ops);
        ops = nullptr;
        if (bar) cudaFree(bar);
        if (strip_done) cudaFree(strip_done);
        if (ctl) cudaFree(ctl);
        for (int g = 0; g < FT_MAX_VRANKS; g++)
            if (peer_opened[g] && peer[g]) cudaIpcCloseMemHandle(peer[g]);
        if (sym && sym_owned) cudaFree(sym);
        bar = nullptr;
        strip_done = nullptr;
        ctl = nullptr;
        sym = nullptr;
        for (int g = 0; g < FT_MAX_VRANKS; g++) {
            peer[g] = nullptr;
            peer_opened[g] = false;
        }
        n_cap = -1;
    }
};

constexpr int kMaxWsplitM = FT_WSPLIT_MAX;
constexpr int64_t kYtopRowsM = 1 << 22;

int mg_alloc(MgRank &R, int n, int G, int rank) {
    R.release();
    CK(cudaGetDevice(&R.dev));
    CK(cudaDeviceGetAttribute(&R.nsm, cudaDevAttrMultiProcessorCount, R.dev));
    R.G = G;
    R.rank = rank;
    R.ldw = ((int64_t)n + 2 + 31) / 32 * 32;
    const int64_t ldw = R.ldw;
    const size_t N1 = (size_t)n + 1;
    cudaError_t e = cudaSuccess;
    auto A = [&](cudaError_t x) {
        if (x != cudaSuccess && e == cudaSuccess) e = x;
    };
    const int ncl_max = (n + 1);  // local columns + r (upper bound)
    A(cudaMalloc(&R.Aw, (size_t)ldw * (ncl_max + 1) * sizeof(double)));
    A(cudaMalloc(&R.V, (size_t)ldw * FT_NBMAX * sizeof(double)));
    A(cudaMalloc(&R.Y, (size_t)ldw * FT_NBMAX * sizeof(double)));
    A(cudaMalloc(&R.T, (size_t)FT_NBMAX * FT_NBMAX * sizeof(double)));
    A(cudaMalloc(&R.Wpart, (size_t)kMaxWsplitM * (N1 + 64) * FT_NBMAX * sizeof(double)));
    A(cudaMalloc(&R.Wt, (N1 + 64) * FT_NBMAX * sizeof(double)));
    A(cudaMalloc(&R.Z, (size_t)ldw * FT_NBMAX * sizeof(double)));
    A(cudaMalloc(&R.bvec, (size_t)4 * ldw * sizeof(double)));
    A(cudaMalloc(&R.acc, (size_t)FT_ACC_SETS * FT_ACC_SET_DOUBLES * sizeof(double)));
    A(cudaMalloc(&R.dpart, (size_t)FT_ACC_SETS * FT_ACC_STRIDE * FT_DPMAX * sizeof(double)));
    A(cudaMalloc(&R.Qr, (size_t)ldw * sizeof(double)));
    A(cudaMalloc(&R.Qc, (size_t)ldw * sizeof(double)));
    A(cudaMalloc(&R.ypart, (size_t)std::min<int64_t>(kYtopRowsM, 64 * N1) * FT_NBMAX * sizeof(double)));
    A(cudaMalloc(&R.rowpart, (size_t)std::min<int64_t>(kYtopRowsM, 64 * N1) * sizeof(double)));
    A(cudaMalloc(&R.vec, (size_t)(ldw + 64) * sizeof(double)));
    A(cudaMalloc(&R.vec2, (size_t)(ldw + 64) * sizeof(double)));
    A(cudaMalloc(&R.bar, 4 * sizeof(unsigned)));
    A(cudaMalloc(&R.strip_done, ((N1 + 63) / 64 + 2) * sizeof(int)));
    A(cudaMalloc(&R.ctl, sizeof(FtCtl)));
    A(cudaMalloc(&R.ck, (size_t)(N1 + N1 + N1 * FT_NBMAX) * sizeof(double)));
    A(cudaMalloc(&R.full, (size_t)(2 * N1 + 8) * sizeof(double)));
    A(cudaMalloc(&R.ops, (size_t)4 * FT_MAX_EVENTS * sizeof(MgOp)));
    R.lay = sym_layout(ldw, G);
    A(cudaMalloc(&R.sym, R.lay.total));
    if (e != cudaSuccess) {
        R.release();
        cudaGetLastError();
        return e == cudaErrorMemoryAllocation ? FT_E_NOMEM : FT_E_CUDA;
    }
    R.sym_owned = true;
    CK(cudaMemset(R.sym, 0, R.lay.total));  // flags start at 0; sequence numbers only grow
    CK(cudaMemset(R.strip_done, 0, ((N1 + 63) / 64 + 2) * sizeof(int)));
    CK(cudaMemset(R.V, 0, (size_t)ldw * FT_NBMAX * sizeof(double)));
    CK(cudaMemset(R.Y, 0, (size_t)ldw * FT_NBMAX * sizeof(double)));
    R.peer[rank] = R.sym;
    R.xseq = 0;
    R.pseq = 0;
    R.n_cap = n;
    return 0;
}

// one exchange over every local rank (xs: the per-rank region descriptions)
int mg_xchg(std::vector<MgRank *> &Rs, int mode, int root, std::vector<XchgRank> xs, cudaStream_t s) {
    XchgLaunch L{};
    L.nr = (int)Rs.size();
    int64_t total = (int64_t)xs[0].rows * xs[0].cols;
    if (total <= 0) return 0;
    for (int q = 0; q < L.nr; q++) {
        MgRank &R = *Rs[q];
        XchgRank x = xs[q];
        x.G = R.G;
        x.rank = R.rank;
        x.mode = mode;
        x.root = root;
        R.xseq++;
        x.seq = R.xseq;
        const int parity = R.xseq & 1;
        if (mode == 0 && total > R.lay.xlen) return FT_E_CUDA;
        for (int g = 0; g < R.G; g++) {
            x.slot_peer[g] = R.xbuf(g, parity);
            x.fl_peer[g] = R.xflags(g);
        }
        L.r[q] = x;
    }
    const int nsm = Rs[0]->nsm;
    int per = (int)std::max<int64_t>(1, std::min<int64_t>((total + 255) / 256, std::max(1, nsm / L.nr)));
    per = std::min(per, FT_FLAG_STRIDE);
    g_ft_launches++;
    void *args[] = {&L};
    CK(cudaLaunchCooperativeKernel((const void *)k_xchg, dim3(per * L.nr), dim3(256), args, 0, s));
    return 0;
}

struct MgCall {
    int n, nb, G, abft, npanels;
    int det = 0;  // opts.deterministic: fixed-order column dots (ranks then agree bitwise)
    double c_thr = 2.0;
    std::vector<ft_fault> faults;  // sites A and C (the owner's words); phases BEFORE_PANEL,
                                   // AFTER_RIGHT, AFTER_UPDATE, AT_END
    std::vector<ft_event> events;
    int detected = 0, corrected = 0, rollbacks = 0, uncorrectable = 0;
    void ev(int kind, int panel, int64_t i, int64_t j, double d) {
        ft_event e;
        e.kind = kind;
        e.panel = panel;
        e.i = i;
        e.j = j;
        e.delta = d;
        events.push_back(e);
    }
    cudaStream_t s;
    std::vector<MgRank *> R;          // local ranks (1 per GPU, or G virtual ranks)
    std::vector<double *> dA, dtau;   // caller slabs / tau per local rank
    int lda;
    int ncl(int rank) const {  // local columns of rank
        int nblk = (n + nb - 1) / nb, c = 0;
        for (int b = rank; b < nblk; b += G) c += std::min(nb, n - b * nb);
        return c;
    }
    int lfirst(int rank, int J) const {  // number of local columns of rank with global index < J
        int c = 0, nblk = (n + nb - 1) / nb;
        for (int b = rank; b < nblk; b += G) {
            int lo = b * nb, hi = std::min(n, lo + nb);
            if (hi <= J) c += hi - lo;
            else if (lo < J) c += J - lo;
        }
        return c;
    }
};

// soft errors on the sharded layout (fault plan): the owner of global column J holds A(:, J) and c(J)
int mg_inject(MgCall &C, int panel, int phase) {
    const int64_t ldw = C.R[0]->ldw;
    for (size_t q = 0; q < C.faults.size() && q < FT_MAXFAULTS; q++) {
        const ft_fault &f = C.faults[q];
        if (f.phase != phase || (phase != FT_PHASE_AT_END && f.panel != panel)) continue;
        if (f.j < 0 || f.j >= C.n) continue;
        const int owner = (int)((f.j / C.nb) % C.G);
        const int64_t l = (f.j / ((int64_t)C.nb * C.G)) * C.nb + f.j % C.nb;
        for (MgRank *R : C.R) {
            if (R->rank != owner) continue;
            double *a = nullptr;
            if (f.site == FT_SITE_A && f.i >= 0 && f.i < C.n) a = R->Aw + f.i + l * ldw;
            else if (f.site == FT_SITE_C) a = R->Aw + C.n + l * ldw;
            if (a) CK(ft_inject(a, (int)q, f.bit, R->ctl, C.s));
        }
    }
    return 0;
}

// the update GEMMs of iteration t on every local rank; sign -1 forward, +1 reverse computation
// (with the retained Y, V, T, W')
int mg_updates(MgCall &C, int t, double sign, bool right) {
    const int n = C.n, nb = C.nb, G = C.G;
    const int64_t ldw = C.R[0]->ldw;
    const int k = t * nb, ib = std::min(nb, n - 2 - k), e = k + ib;
    const int owner = t % G, lk = (t / G) * nb;
    for (MgRank *Rp : C.R) {
        MgRank &R = *Rp;
        const int ncl = C.ncl(R.rank);
        const int le = C.lfirst(R.rank, e);
        GemmRightParams g{};
        g.A = R.Aw;
        g.lda = ldw;
        g.ldw = ldw;
        g.Y = R.Y;
        g.V = R.V;
        g.K = ib;
        g.sign = sign;
        g.Wpart = R.Wpart;
        g.wsplit_stride = ((int64_t)n + 1 + 64) * FT_NBMAX;
        g.ctl = sign < 0 ? R.ctl : nullptr;
        g.has_m = R.rank == owner ? 1 : 0;
        g.m_r_hi = k + 1;
        g.m_c_lo = lk + 1;
        g.m_c_hi = lk + ib;
        g.do_right = 1;
        g.r_lo = 0;
        g.r_hi = C.abft ? n + 1 : n;
        g.c_lo = le;
        g.c_hi = ncl + (C.abft ? 1 : 0);
        g.wr_lo = k + 1;
        g.wr_hi = n;
        g.do_w = sign < 0 ? 1 : 0;
        g.nsplit = ft_gemm_splits(g.r_lo, g.r_hi, g.c_lo, g.c_hi, R.nsm);
        if (g.do_w) {
            g.Wt = R.Wt;
            g.T = R.T;
            g.transT = 1;
            g.strip_done = R.strip_done;
        }
        g.cm_G = G;
        g.cm_rank = R.rank;
        g.cm_nb = nb;
        g.cm_ncl = ncl;
        g.cm_n = n;
        GemmLeftParams h{};
        h.A = R.Aw;
        h.lda = ldw;
        h.ldw = ldw;
        h.V = R.V;
        h.T = R.T;
        h.Wpart = R.Wpart;
        h.Wt = R.Wt;
        h.r_lo = k + 1;
        h.r_hi = C.abft ? n + 1 : n;
        h.c_lo = le;
        h.c_hi = g.c_hi;
        h.K = ib;
        h.nsplit = g.nsplit;
        h.wsplit_stride = g.wsplit_stride;
        h.transT = 1;
        h.sign = sign;
        h.ctl = sign < 0 ? R.ctl : nullptr;
        h.wt_ready = 1;
        h.endcheck = 0;
        h.n = n;
        if (right) CK(ft_launch_gemm_right(g, C.s));
        else if (g.c_hi > g.c_lo) CK(ft_launch_gemm_left(h, C.s));
    }
    return 0;
}

// one iteration on every local rank (Alg. 3 on the sharded layout)
int mg_panel(MgCall &C, int t) {
    const int n = C.n, nb = C.nb, G = C.G;
    const int nr = (int)C.R.size();
    cudaStream_t s = C.s;
    const int64_t ldw = C.R[0]->ldw;
    const int gr = ft_panel_group_rows();
    const int k = t * nb, ib = std::min(nb, n - 2 - k), e = k + ib;
    const int owner = t % G, lk = (t / G) * nb;
    if (C.abft) {
        if (mg_inject(C, t, FT_PHASE_BEFORE_PANEL)) return FT_E_CUDA;
        for (MgRank *R : C.R) {  // diskless checkpoint: r, kappa, own c, the owner's panel
            g_ft_launches++;
            k_mg_ckpt<<<std::max(1, std::min((int)((n + 1) * (int64_t)ib / 256) + 1, 2 * R->nsm)), 256, 0, s>>>(
                R->Aw, ldw, n, C.ncl(R->rank), lk, ib, R->rank == owner, R->ck, 0, R->ctl);
            CK(cudaGetLastError());
        }
    }
    // 1. owner's panel columns (rows 0..n) -> every rank's P
    for (int q = 0; q < nr; q++)
        if (G > 1 && C.R[q]->rank == owner)
            CK(mg_copy(C.R[q]->Aw + (int64_t)lk * ldw, ldw, C.R[q]->P(), ldw, n + 1, ib, s, C.R[q]->ctl));
    if (G > 1) {
        std::vector<XchgRank> xs(nr);
        for (int q = 0; q < nr; q++) {
            MgRank &R = *C.R[q];
            xs[q] = XchgRank{};
            xs[q].src = R.P();
            xs[q].ld = ldw;
            xs[q].rows = n + 1;
            xs[q].cols = ib;
            xs[q].ctl = R.ctl;
            for (int g = 0; g < G; g++) xs[q].dst_peer[g] = reinterpret_cast<double *>(R.peer[g] + R.lay.P);
        }
        if (mg_xchg(C.R, 1, owner, xs, s)) return FT_E_CUDA;
    }
    // 2. the panel (every rank, one multi-rank launch)
    PanelLaunch L{};
    L.nr = nr;
    for (int q = 0; q < nr; q++) {
        MgRank &R = *C.R[q];
        PanelParams &p = L.r[q];
        p = PanelParams{};
        p.A = R.Aw;
        p.ldw = ldw;
        p.V = R.V;
        p.Y = R.Y;
        p.T = R.T;
        p.tau = C.dtau[q];
        p.bvec = R.bvec;
        p.Z = R.Z;
        p.acc = R.acc;
        p.dpart = C.det ? R.dpart : nullptr;
        p.bar = R.bar + (t & 1);
        p.bar_next = R.bar + ((t + 1) & 1);
        p.ctl = R.ctl;
        p.Qr = R.Qr;
        p.Qc = R.Qc;
        p.n = n;
        p.ihi = n;
        p.k = k;
        p.ib = ib;
        p.abft = C.abft;
        p.verify = 0;
        p.rbase = ((k + 1) / gr) * gr;
        const int rendp = ((C.abft ? n + 1 : n) + gr - 1) / gr * gr;
        p.ngroups = (rendp - p.rbase) / gr;
        p.Apan = G > 1 ? R.P() - (int64_t)k * ldw : R.Aw;  // one rank: the panel in place
        const int ncl = C.ncl(R.rank);
        p.rcol = R.Aw + (int64_t)ncl * ldw;
        p.G = G;
        p.rank = R.rank;
        p.cbnb = nb;
        p.owner = R.rank == owner;
        p.lcol0 = C.lfirst(R.rank, e);
        p.lcol1 = ncl;
        p.e = e;
        p.yx = R.yx(R.rank);
        for (int g = 0; g < G; g++) {
            p.ypeer[g] = R.yx(g);
            p.fpeer[g] = R.flags(g);
        }
        p.flags = R.flags(R.rank);
        p.seq0 = R.pseq;
    }
    CK(ft_launch_panel_multi(L, C.R[0]->nsm, s));
    // 3. owner: P -> own panel columns
    for (int q = 0; q < nr; q++)
        if (G > 1 && C.R[q]->rank == owner)
            CK(mg_copy(C.R[q]->P(), ldw, C.R[q]->Aw + (int64_t)lk * ldw, ldw, n + 1, ib, s, C.R[q]->ctl));
    // 4. Y_top partial per rank, then summed across ranks
    for (int q = 0; q < nr; q++) {
        MgRank &R = *C.R[q];
        const int ncl = C.ncl(R.rank);
        YtopParams y{};
        y.A = R.Aw;
        y.ldw = ldw;
        y.V = R.V;
        y.T = R.T;
        y.Y = R.Y;
        y.ypart = R.ypart;
        y.rowpart = R.rowpart;
        y.ctl = R.ctl;
        y.n = n;
        y.ihi = n;
        y.k = k;
        y.ib = ib;
        y.abft = C.abft;
        y.verify = 0;
        y.decide = 0;
        y.panel = t;
        y.cm_G = G;
        y.cm_rank = R.rank;
        y.cm_nb = nb;
        y.cm_ncl = ncl;
        y.kc0 = C.lfirst(R.rank, k + 1);
        y.kc1 = ncl;
        const int nm = (k + 1 + ft_ytop_rows_per_cta() - 1) / ft_ytop_rows_per_cta();
        const int nkt = (y.kc1 - y.kc0 + 31) / 32;
        int ns = std::max(1, std::min({(2 * R.nsm) / nm, std::max(nkt / 2, 1), 64}));
        while ((int64_t)ns * (k + 1) > kYtopRowsM) ns--;
        y.nsplit = std::max(ns, 1);
        if (y.kc1 > y.kc0) {
            CK(ft_launch_ytop(y, s));
        } else {  // no own columns right of the panel: a zero partial (halt-aware: Y is kept for a rollback)
            for (int j = 0; j < ib; j++) CK(ft_zero_if_running(R.Y + (int64_t)j * ldw, (size_t)k + 1, R.ctl, s));
        }
    }
    {
        std::vector<XchgRank> xs(nr);
        for (int q = 0; q < nr; q++) {
            xs[q] = XchgRank{};
            xs[q].src = C.R[q]->Y;
            xs[q].ld = ldw;
            xs[q].rows = k + 1;
            xs[q].cols = ib;
            xs[q].ctl = C.R[q]->ctl;
        }
        if (mg_xchg(C.R, 0, 0, xs, s)) return FT_E_CUDA;
    }
    // 5./6. rank-local right (+W, +M on the owner) and left updates
    if (mg_updates(C, t, -1.0, true)) return FT_E_CUDA;
    if (C.abft && mg_inject(C, t, FT_PHASE_AFTER_RIGHT)) return FT_E_CUDA;
    if (mg_updates(C, t, -1.0, false)) return FT_E_CUDA;
    if (C.abft) {
        if (mg_inject(C, t, FT_PHASE_AFTER_UPDATE)) return FT_E_CUDA;
        // end of iteration (Alg. 3 l.12-13): the sums, rank-ordered allreduce, the same decision everywhere
        for (MgRank *R : C.R) {
            g_ft_launches++;
            k_mg_endsums<<<1, 256, 0, s>>>(R->Aw, ldw, n, C.ncl(R->rank), R->rank, R->vec, R->ctl);
            CK(cudaGetLastError());
        }
        std::vector<XchgRank> xs(nr);
        for (int q = 0; q < nr; q++) {
            xs[q] = XchgRank{};
            xs[q].src = C.R[q]->vec;
            xs[q].ld = 3;
            xs[q].rows = 3;
            xs[q].cols = 1;
            xs[q].ctl = C.R[q]->ctl;
        }
        if (mg_xchg(C.R, 0, 0, xs, s)) return FT_E_CUDA;
        for (MgRank *R : C.R) {
            g_ft_launches++;
            k_mg_decide<<<1, 1, 0, s>>>(R->vec, n, t, R->ctl);
            CK(cudaGetLastError());
        }
    }
    return 0;
}

// distributed location and correction: row sums of the logical matrix summed across
// ranks, every rank's column discrepancies gathered, the same R12 plan on every rank, each fix
// applied by the owner of its column (row form A(i,j) += D_r(i), column form A(i,j) += D_c(j)),
// r / kappa refreshed on every rank, c on its owner; then re-verified.  cdone: finished columns.
int mg_verify_correct(MgCall &C, int panel, int cdone, bool *clean) {
    const int n = C.n, nb = C.nb, G = C.G;
    const int nr = (int)C.R.size();
    cudaStream_t s = C.s;
    const int64_t ldw = C.R[0]->ldw;
    *clean = true;
    for (int pass = 0; pass < 2; pass++) {
        for (MgRank *R : C.R) {
            const int ncl = C.ncl(R->rank);
            CK(cudaMemsetAsync(R->full, 0, (size_t)(2 * n + 3) * sizeof(double), s));
            g_ft_launches += 3;
            k_mg_verify_local<<<std::max(1, std::min((n + 255) / 256, 2 * R->nsm)), 256, 0, s>>>(
                R->Aw, ldw, n, ncl, G, R->rank, nb, R->full, R->vec2, cdone);
            k_mg_scatter_dc<<<std::max(1, (ncl + 255) / 256), 256, 0, s>>>(R->vec2, ncl, G, R->rank, nb, n, R->full + n);
            k_mg_endsums<<<1, 256, 0, s>>>(R->Aw, ldw, n, ncl, R->rank, R->full + 2 * n, R->ctl);
            CK(cudaGetLastError());
        }
        std::vector<XchgRank> xs(nr);
        for (int q = 0; q < nr; q++) {
            xs[q] = XchgRank{};
            xs[q].src = C.R[q]->full;
            xs[q].ld = 2 * n + 3;
            xs[q].rows = 2 * n + 3;
            xs[q].cols = 1;
        }
        if (mg_xchg(C.R, 0, 0, xs, s)) return FT_E_CUDA;
        MgRank &R0 = *C.R[0];
        std::vector<double> buf(2 * n + 3), r(n + 1);
        FtCtl h;
        CK(cudaMemcpyAsync(buf.data(), R0.full, (2 * n + 3) * sizeof(double), cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(r.data(), R0.Aw + (int64_t)C.ncl(R0.rank) * ldw, (n + 1) * sizeof(double),
                           cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(&h, R0.ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        const double tau = C.c_thr * n * kEpsM * h.normF;
        std::vector<double> Dr(n), Dc(buf.begin() + n, buf.begin() + 2 * n);
        for (int i = 0; i < n; i++) Dr[i] = r[i] - buf[i];
        const double Sr = buf[2 * n], Sc = buf[2 * n + 1], kap = buf[2 * n + 2];
        std::vector<FtFix> fx;
        const int st = ft_host_decode(n, Dr.data(), Dc.data(), Sr - kap, Sc - kap, tau, &fx);
        if (pass == 1) {
            if (st != 0) {
                C.ev(FT_EV_UNCORRECTABLE, panel, -1, -1, 0.0);
                C.uncorrectable++;
                return FT_E_UNCORRECTABLE;
            }
            C.corrected++;
            return 0;
        }
        if (st == 0) return 0;
        *clean = false;
        int nrf = 0, ncf = 0;
        for (int i = 0; i < n; i++) {
            nrf += !(std::fabs(Dr[i]) <= tau);
            ncf += !(std::fabs(Dc[i]) <= tau);
        }
        C.ev(FT_EV_DETECT, panel, nrf, ncf, 0.0);
        C.detected++;
        if (st == 2) {
            C.ev(FT_EV_UNCORRECTABLE, panel, nrf, ncf, 0.0);
            C.uncorrectable++;
            return FT_E_UNCORRECTABLE;
        }
        // per-rank op lists (the same plan everywhere)
        for (MgRank *R : C.R) {
            std::vector<MgOp> ops;
            for (const FtFix &f : fx) {
                MgOp o{};
                if (f.kind == 0 || f.kind == 1 || f.kind == 3) {  // data (row / column form), c(j)
                    const int J = (int)f.j;
                    if ((J / nb) % G != R->rank) continue;
                    o.l = (J / ((int64_t)nb * G)) * nb + J % nb;
                    o.i = f.i;
                    o.kind = f.kind == 3 ? 2 : 0;
                    o.v = f.kind == 0 ? Dr[f.i] : (f.kind == 1 ? Dc[J] : -Dc[J]);
                } else if (f.kind == 2) {  // r(i) = the row sum (every rank's copy)
                    o.i = f.i;
                    o.kind = 1;
                    o.v = buf[f.i];
                } else {  // kappa = sum r
                    o.kind = 3;
                    double sr = 0.0;
                    for (int i = 0; i < n; i++) sr += r[i];
                    o.v = sr;
                }
                ops.push_back(o);
            }
            if (ops.empty()) continue;
            const int m = (int)std::min<size_t>(ops.size(), 4 * FT_MAX_EVENTS);
            CK(cudaMemcpyAsync(R->ops, ops.data(), m * sizeof(MgOp), cudaMemcpyHostToDevice, s));
            g_ft_launches++;
            k_mg_apply<<<std::max(1, (m + 255) / 256), 256, 0, s>>>(R->Aw, ldw, n, C.ncl(R->rank),
                                                                     reinterpret_cast<const MgOp *>(R->ops), m);
            CK(cudaGetLastError());
            CK(cudaStreamSynchronize(s));
        }
        for (const FtFix &f : fx) {
            const int kind = f.kind <= 1 ? FT_EV_FIX_DATA : f.kind == 2 ? FT_EV_FIX_R : f.kind == 3 ? FT_EV_FIX_C
                                                                                                     : FT_EV_FIX_K;
            const double d = f.kind == 0 ? Dr[f.i] : f.kind == 1 ? Dc[f.j] : f.kind == 2 ? -Dr[f.i]
                             : f.kind == 3 ? -Dc[f.j] : 0.0;
            C.ev(kind, panel, f.i, f.j, d);
        }
    }
    return 0;
}

int mg_run(MgCall &C, ft_report *rep) {
    const int n = C.n, G = C.G;
    const int nr = (int)C.R.size();
    cudaStream_t s = C.s;
    const int64_t ldw = C.R[0]->ldw;
    cudaEvent_t ev0, ev1;
    CK(cudaEventCreate(&ev0));
    CK(cudaEventCreate(&ev1));
    CK(cudaEventRecord(ev0, s));
    // ---- start: copy in, encode (a1) ----
    for (int q = 0; q < nr; q++) {
        MgRank &R = *C.R[q];
        const int ncl = C.ncl(R.rank);
        CK(ft_ctl_init(R.ctl, C.c_thr, s));
        CK(cudaMemsetAsync(R.Aw, 0, (size_t)ldw * (ncl + 1) * sizeof(double), s));
        CK(cudaMemsetAsync(R.V, 0, (size_t)ldw * FT_NBMAX * sizeof(double), s));
        CK(cudaMemsetAsync(R.Y, 0, (size_t)ldw * FT_NBMAX * sizeof(double), s));
        CK(cudaMemsetAsync(R.bvec, 0, (size_t)4 * ldw * sizeof(double), s));
        CK(cudaMemsetAsync(R.bar, 0, 4 * sizeof(unsigned), s));
        CK(cudaMemsetAsync(R.acc, 0, (size_t)FT_ACC_SETS * FT_ACC_SET_DOUBLES * sizeof(double), s));
        CK(cudaMemsetAsync(R.Qr, 0, ldw * sizeof(double), s));
        CK(cudaMemsetAsync(R.Qc, 0, ldw * sizeof(double), s));
        if (n > 1) CK(cudaMemsetAsync(C.dtau[q], 0, (n - 1) * sizeof(double), s));
        CK(mg_copy(C.dA[q], C.lda, R.Aw, ldw, n, ncl, s));
        if (C.abft) {
            g_ft_launches += 3;
            if (ncl > 0) k_mg_encode_cols<<<ncl, 256, 0, s>>>(R.Aw, ldw, n, ncl, R.vec2);
            k_mg_rowsums<<<std::max(1, std::min((n + 255) / 256, 4 * R.nsm)), 256, 0, s>>>(R.Aw, ldw, n, ncl, R.vec);
            k_mg_frob<<<1, 32, 0, s>>>(R.vec2, ncl, R.vec + n);
            CK(cudaGetLastError());
        }
    }
    if (C.abft) {
        std::vector<XchgRank> xs(nr);
        for (int q = 0; q < nr; q++) {
            xs[q] = XchgRank{};
            xs[q].src = C.R[q]->vec;
            xs[q].ld = n + 1;
            xs[q].rows = n + 1;  // row sums + ||A||_F^2
            xs[q].cols = 1;
        }
        if (mg_xchg(C.R, 0, 0, xs, s)) return FT_E_CUDA;
        for (int q = 0; q < nr; q++) {
            MgRank &R = *C.R[q];
            g_ft_launches++;
            k_mg_encode_finish<<<1, 256, 0, s>>>(R.Aw, ldw, n, C.ncl(R.rank), R.vec, R.ctl);
            CK(cudaGetLastError());
        }
    }
    // ---- panels, with the halt protocol: a failed end check halts every rank identically; the
    // host then rolls the iteration back, locates, corrects and redoes it ----
    int info = 0, t0 = 0, attempts = 0;
    while (true) {
        for (int t = t0; t < C.npanels; t++) {
            const int rc = mg_panel(C, t);
            if (rc) return rc;
        }
        if (!C.abft) break;
        FtCtl h;
        CK(cudaMemcpyAsync(&h, C.R[0]->ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (!h.halt) break;
        if (++attempts > 4 * (C.npanels + 1) + (int)C.faults.size() * 4) {
            C.ev(FT_EV_UNCORRECTABLE, h.halt_panel, -1, -1, 0.0);
            C.uncorrectable++;
            info = FT_E_UNCORRECTABLE;
            break;
        }
        const int t = h.halt_panel, k = t * C.nb, ib = std::min(C.nb, n - 2 - k);
        const int owner = t % G, lk = (t / G) * C.nb;
        int zero = 0;
        for (MgRank *R : C.R) {
            CK(cudaMemcpyAsync(&R->ctl->halt, &zero, sizeof(int), cudaMemcpyHostToDevice, s));
            R->pseq += (unsigned)n + 1u;  // the redone panel's exchange flags must be new values
            // the panel kernels' grid-barrier counters and reduction sets start from zero again
            CK(cudaMemsetAsync(R->bar, 0, 4 * sizeof(unsigned), s));
            CK(cudaMemsetAsync(R->acc, 0, (size_t)FT_ACC_SETS * FT_ACC_SET_DOUBLES * sizeof(double), s));
        }
        // reverse computation: add back the left, then the right update
        if (mg_updates(C, t, +1.0, false) || mg_updates(C, t, +1.0, true)) return FT_E_CUDA;
        C.ev(FT_EV_ROLLBACK, t, h.halt_reason, 0, 0.0);
        C.rollbacks++;
        for (MgRank *R : C.R) {  // restore the checkpoint
            g_ft_launches++;
            k_mg_ckpt<<<std::max(1, std::min((int)((n + 1) * (int64_t)ib / 256) + 1, 2 * R->nsm)), 256, 0, s>>>(
                R->Aw, ldw, n, C.ncl(R->rank), lk, ib, R->rank == owner, R->ck, 1, R->ctl);
            CK(cudaGetLastError());
        }
        bool clean = true;
        const int r1 = mg_verify_correct(C, t, k, &clean);
        if (r1 == FT_E_UNCORRECTABLE) {
            info = r1;
            break;
        }
        if (r1) return r1;
        t0 = t;
    }
    for (int q = 0; q < nr; q++) C.R[q]->pseq += (unsigned)n + 1u;
    // ---- final verification (a12) with correction ----
    if (C.abft && info == 0) {
        if (mg_inject(C, -1, FT_PHASE_AT_END)) return FT_E_CUDA;
        bool clean = true;
        const int r1 = mg_verify_correct(C, -1, n - 1, &clean);
        if (r1 == FT_E_UNCORRECTABLE) info = r1;
        else if (r1) return r1;
    }
    for (int q = 0; q < nr; q++) CK(mg_copy(C.R[q]->Aw, ldw, C.dA[q], C.lda, n, C.ncl(C.R[q]->rank), s));
    CK(cudaEventRecord(ev1, s));
    CK(cudaStreamSynchronize(s));
    float ms = 0.f;
    cudaEventElapsedTime(&ms, ev0, ev1);
    cudaEventDestroy(ev0);
    cudaEventDestroy(ev1);
    if (rep) {
        memset(rep, 0, sizeof(*rep));
        std::vector<ft_event> all;
        for (size_t q = 0; q < C.faults.size() && q < FT_MAXFAULTS; q++) {
            const ft_fault &f = C.faults[q];
            const int owner = (int)((f.j / C.nb) % G);
            for (MgRank *R : C.R) {
                if (R->rank != owner) continue;
                FtCtl h;
                CK(cudaMemcpy(&h, R->ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost));
                if (!h.inj_done[q]) continue;
                ft_event e;
                e.kind = FT_EV_INJECT;
                e.panel = f.phase == FT_PHASE_AT_END ? -1 : f.panel;
                e.i = f.i;
                e.j = f.j;
                e.delta = h.inj_delta[q];
                all.push_back(e);
            }
        }
        all.insert(all.end(), C.events.begin(), C.events.end());
        rep->nevents = (int)std::min<size_t>(all.size(), FT_MAX_EVENTS);
        for (int q = 0; q < rep->nevents; q++) rep->events[q] = all[q];
        rep->detected = C.detected;
        rep->corrected = C.corrected;
        rep->rollbacks = C.rollbacks;
        rep->uncorrectable = C.uncorrectable;
        FtCtl h;
        CK(cudaMemcpy(&h, C.R[0]->ctl, sizeof(FtCtl), cudaMemcpyDeviceToHost));
        double drift;
        memcpy(&drift, &h.drift_bits, 8);
        rep->max_drift_rel = drift;
        rep->ms[0] = ms;
        for (int q = 1; q < 8; q++) rep->ms[q] = -1.0;
    }
    return info;
}

int mg_validate(int n, int ilo, int ihi, int lda, int nranks, const ft_opts &o) {
    if (n < 0) return -1;
    if (ilo != 1) return -2;                   // round 1: full reduction only
    if (ihi != n) return -3;
    if (nranks < 1 || nranks > FT_MAX_VRANKS) return -9;
    if (lda < std::max(1, n)) return -5;
    if (o.nb < 0 || o.nb > FT_NBMAX) return -7;
    if (o.abft != 0 && o.abft != 1) return -7;
    if (o.stop_after_panel != -1 || o.weighted != 0) return -7;  // single-GPU path only
    if (o.deterministic != 0 && o.deterministic != 1) return -7;
    if (o.nfaults < 0 || o.nfaults > FT_MAXFAULTS || (o.nfaults > 0 && (!o.faults || !o.abft))) return -7;
    for (int q = 0; q < o.nfaults; q++) {
        const ft_fault &f = o.faults[q];
        // soft errors in words with one owner: A and its column checksum c (the replicated r, kappa and
        // the redundantly computed V, Y, T are per-rank copies: their faults are out of scope here)
        if (f.site != FT_SITE_A && f.site != FT_SITE_C) return -7;
        if (f.phase == FT_PHASE_AFTER_PANEL) return -7;
    }
    return 0;
}

// virtual ranks on this device (tests / one-GPU measurements)
std::vector<MgRank> g_vranks;
// the real rank of this process
MgRank g_rank;

}  // namespace

extern "C" {

int ft_dgehrd_vranks(int n, int ilo, int ihi, double *const *dA_local, int lda_local, double *const *dtau,
                     int nranks, const ft_opts *opts) {
    std::lock_guard<std::recursive_mutex> api_lock(ft_api_mutex());
    ft_opts o;
    ft_opts_default(&o);
    if (opts) o = *opts;
    int info = mg_validate(n, ilo, ihi, lda_local, nranks, o);
    if (info) return info;
    if (!dA_local || !dtau) return -4;
    if (n < 3) return ft_dgehrd(n, ilo, ihi, dA_local[0], lda_local, dtau[0], opts);  // nothing to shard
    int dev = 0;
    CK(cudaGetDevice(&dev));
    if ((int)g_vranks.size() != nranks || g_vranks[0].n_cap < n || g_vranks[0].dev != dev) {
        for (auto &R : g_vranks) R.release();
        g_vranks.clear();
        g_vranks.resize(nranks);
        for (int q = 0; q < nranks; q++) {
            int rc = mg_alloc(g_vranks[q], n, nranks, q);
            if (rc) return rc;
        }
        for (int q = 0; q < nranks; q++)
            for (int g = 0; g < nranks; g++) g_vranks[q].peer[g] = g_vranks[g].sym;
    }
    MgCall C;
    C.n = n;
    C.nb = o.nb > 0 ? o.nb : (n < 4096 ? 32 : 64);
    C.G = nranks;
    C.abft = o.abft;
    C.det = o.deterministic;
    C.npanels = (n - 2 + C.nb - 1) / C.nb;
    C.s = (cudaStream_t)o.stream;
    C.lda = lda_local;
    for (int q = 0; q < nranks; q++) {
        C.R.push_back(&g_vranks[q]);
        C.dA.push_back(dA_local[q]);
        C.dtau.push_back(dtau[q]);
    }
    C.c_thr = o.c_thr > 0 ? o.c_thr : 2.0;
    for (int q = 0; q < o.nfaults; q++) C.faults.push_back(o.faults[q]);
    return mg_run(C, o.report);
}

int ft_mgpu_setup(int n_max, int rank, int nranks, ft_ipc_handle *handle_out) {
    std::lock_guard<std::recursive_mutex> api_lock(ft_api_mutex());
    if (nranks < 1 || nranks > FT_MAX_VRANKS || rank < 0 || rank >= nranks || n_max < 0 || !handle_out) return -9;
    int rc = mg_alloc(g_rank, std::max(n_max, 3), nranks, rank);
    if (rc) return rc;
    cudaIpcMemHandle_t h;
    CK(cudaIpcGetMemHandle(&h, g_rank.sym));
    static_assert(sizeof(cudaIpcMemHandle_t) <= sizeof(handle_out->bytes), "ipc handle size");
    memset(handle_out->bytes, 0, sizeof(handle_out->bytes));
    memcpy(handle_out->bytes, &h, sizeof(h));
    return 0;
}

int ft_mgpu_connect(const ft_ipc_handle *handles, int rank, int nranks) {
    std::lock_guard<std::recursive_mutex> api_lock(ft_api_mutex());
    if (!handles || g_rank.n_cap < 0 || nranks != g_rank.G || rank != g_rank.rank) return -9;
    for (int g = 0; g < nranks; g++) {
        if (g == rank) continue;
        cudaIpcMemHandle_t h;
        memcpy(&h, handles[g].bytes, sizeof(h));
        void *p = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {  // a peer on the same device: no peer access to enable
            if (getenv("FT_DEBUG")) fprintf(stderr, "ftgehrd: cudaIpcOpenMemHandle (lazy peer access): %s\n", cudaGetErrorString(e));
            cudaGetLastError();
            e = cudaIpcOpenMemHandle(&p, h, 0);
        }
        if (e != cudaSuccess && getenv("FT_DEBUG")) fprintf(stderr, "ftgehrd: cudaIpcOpenMemHandle: %s\n", cudaGetErrorString(e));
        CK(e);
        g_rank.peer[g] = reinterpret_cast<char *>(p);
        g_rank.peer_opened[g] = true;
    }
    return 0;
}

int ft_dgehrd_mgpu(int n, int ilo, int ihi, double *dA_local, int lda_local, double *dtau, int rank, int nranks,
                   const ft_opts *opts) {
    std::lock_guard<std::recursive_mutex> api_lock(ft_api_mutex());
    ft_opts o;
    ft_opts_default(&o);
    if (opts) o = *opts;
    if (nranks == 1) return ft_dgehrd(n, ilo, ihi, dA_local, lda_local, dtau, opts);
    int info = mg_validate(n, ilo, ihi, lda_local, nranks, o);
    if (info) return info;
    if (rank < 0 || rank >= nranks) return -8;
    if (!dA_local || !dtau) return -4;
    if (g_rank.n_cap < n || g_rank.G != nranks || g_rank.rank != rank) return -9;  // ft_mgpu_setup/connect first
    for (int g = 0; g < nranks; g++)
        if (!g_rank.peer[g]) return -9;
    MgCall C;
    C.n = n;
    C.nb = o.nb > 0 ? o.nb : (n < 4096 ? 32 : 64);
    C.G = nranks;
    C.abft = o.abft;
    C.det = o.deterministic;
    C.npanels = (n - 2 + C.nb - 1) / C.nb;
    C.s = (cudaStream_t)o.stream;
    C.lda = lda_local;
    C.R.push_back(&g_rank);
    C.dA.push_back(dA_local);
    C.dtau.push_back(dtau);
    C.c_thr = o.c_thr > 0 ? o.c_thr : 2.0;
    for (int q = 0; q < o.nfaults; q++) C.faults.push_back(o.faults[q]);
    return mg_run(C, o.report);
}

// IPC bootstrap probe (tests: two processes on one device, no persistent kernel): put writes v into
// slot `rank` of every peer's symmetric region through its CUDA IPC mapping; get reads the own slots
int ft_mgpu_probe_put(double v) {
    if (g_rank.n_cap < 0) return -9;
    for (int g = 0; g < g_rank.G; g++) {
        if (!g_rank.peer[g]) return -9;
        CK(cudaMemcpy(g_rank.peer[g] + g_rank.lay.P + (size_t)g_rank.rank * sizeof(double), &v, sizeof(double),
                      cudaMemcpyHostToDevice));
    }
    CK(cudaDeviceSynchronize());
    return 0;
}
int ft_mgpu_probe_get(double *out) {
    if (g_rank.n_cap < 0 || !out) return -9;
    CK(cudaMemcpy(out, g_rank.sym + g_rank.lay.P, (size_t)g_rank.G * sizeof(double), cudaMemcpyDeviceToHost));
    return 0;
}

void ft_mgpu_finalize(void) {
    for (auto &R : g_vranks) R.release();
    g_vranks.clear();
    g_rank.release();
}

}  // extern "C"
