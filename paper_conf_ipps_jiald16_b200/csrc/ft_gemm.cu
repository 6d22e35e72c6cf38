// ft_gemm.cu -- FP64 tensor-core (DMMA) block-reflector updates on the augmented matrix.
//
// Right update (Alg. 3 l.8/l.10; Fig. 4c-d):  A_aug(rows, cols) -= Y_aug V_aug(cols,:)^T
// fused with W = V^T A_new (the first half of the left update, DLARFB 'L','T' P:42/P:56 l.8),
// and the left update (Alg. 3 l.11, Fig. 4e):         A_aug(rows, cols) -= V_aug (T^T W).
// Row n of Y_aug/V_aug is Y_chk / V_chk and column n of A_aug is the row checksum r, row n
// the column checksum c -- so Theorem 1 is carried by the same tiles.
// Rollback (reverse computation, Alg. 3 l.14) is the same kernels with sign +1.
//
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include <cuda.h>
#include <cudaTypedefs.h>

#include "ft_common.cuh"
#include "ft_internal.h"

// Tiling (both kernels): a CTA owns a 64-column strip and a contiguous range of 64-row
// tiles.  The MMA is formulated on the transpose, D = C^T (cols x rows), so that an
// accumulator fragment holds two CONSECUTIVE rows of one column: the C tile moves between
// HBM and the DMMA accumulators with 16-byte vector loads/stores and never touches shared
// memory.  The small operands (V, Y, W') are k-major cp.async tiles in shared memory with
// a stride of 68 doubles (= 4 mod 16: every fragment load is bank-conflict free).
//   right:  D(cols, rows) += V(cols, :) Y(rows, :)^T,  then  W^T(cols, :) += C_new^T V(rows, :)
//           -- C_new^T as the A operand comes from the accumulators by an in-warp shuffle
//   left:   D(cols, rows) += W'^T(cols, :) V(rows, :)^T
// W partials are written per row split and summed (with op(T)) by k_wprep, so every pass
// is deterministic.
#define UB 64   // tile rows / strip columns
#define UT 256  // threads (8 warps)
#define SK 68   // smem stride of the k-major operand tiles

// Row splits per strip: minimise waves * tiles-per-CTA for per_sm resident CTAs per SM
// (the grid is nstrip x ns CTAs; a ragged last wave idles SMs).
// ovh: fixed per-CTA cost (prologue: operand strip load, pipeline fill) in quarter tiles
static int best_splits(int nstrip, int nrt, int nsm, int cap, int per_sm, int ovh = 0) {
    const int slots = per_sm * nsm;
    int best = 1;
    long long best_cost = -1;
    for (int ns = 1; ns <= cap && ns <= nrt; ns++) {
        const long long waves = ((long long)nstrip * ns + slots - 1) / slots;
        const long long cost = waves * (4 * ((nrt + ns - 1) / ns) + ovh);
        if (best_cost < 0 || cost < best_cost) {
            best_cost = cost;
            best = ns;
        }
    }
    return best;
}
// Right-update tile weights: a tile above the W rows (rows < wr_lo: the rows 0..k the update
// reaches but W = V^T A_new does not) runs the right pass only and counts 1; a tile that also runs
// the W pass counts 2 (twice the DMMA work, the same HBM traffic).  The row splits of a strip cut
// it into equal WEIGHTS (the kernel maps split y to its tiles with right_split_tile), so at late
// panels -- where most rows are above the panel -- the CTAs holding W tiles are no longer the tail.
// tw: the number of right-only tiles at the top of the strip (nrt: none takes part in W).
__host__ __device__ inline int right_split_tile(long long u, int tw) {
    return u <= tw ? (int)u : tw + (int)((u - tw + 1) / 2);
}
static inline int right_tw(int wr_lo, int rbase, int nrt) {
    if (wr_lo < 0) return 0;
    const int t = (wr_lo - rbase) / UB;
    return t < 0 ? 0 : (t > nrt ? nrt : t);
}
int ft_gemm_splits(int r_lo, int r_hi, int c_lo, int c_hi, int nsm, int extra_strips, int wr_lo) {
    // extra_strips: strips of the same launch outside [c_lo, c_hi) (the M-part strip); they take
    // grid slots like the others (counted as full strips: the model stays an upper bound)
    const int nstrip = (c_hi - c_lo + UB - 1) / UB + extra_strips;
    const int rbase = (r_lo / UB) * UB;
    const int nrt = (r_hi - rbase + UB - 1) / UB;
    // right update: one CTA per SM (the next C tile is prefetched in registers)
    // per-CTA prologue / epilogue (V strip, first copies, W partials) of 1.5 tiles: with the split cap
    // at 32 a zero term picks many short CTAs (right update at C3: 356 ms at 0, 340 ms at 3-10;
    // profiles/r02/gemm_tma/right_ovh_sweep.txt); FT_RIGHT_OVH overrides for sweeps
    static const int ovh = getenv("FT_RIGHT_OVH") ? atoi(getenv("FT_RIGHT_OVH")) : 6;
    if (nstrip <= 0 || nrt <= 0) return 1;
    const int tw = right_tw(wr_lo, rbase, nrt);
    const long long units = (long long)tw + 2LL * (nrt - tw);  // weights: right-only 1, right + W 2
    const int slots = nsm;
    int best = 1;
    long long best_cost = -1;
    for (int ns = 1; ns <= FT_WSPLIT_MAX && ns <= nrt; ns++) {
        const long long waves = ((long long)nstrip * ns + slots - 1) / slots;
        // heaviest split in quarter tiles (a right-only tile is half a right + W tile = 2 quarters)
        long long umax = 0;
        for (int y = 0; y < ns; y++) {
            const long long u0 = (long long)y * units / ns, u1 = (long long)(y + 1) * units / ns;
            const int a = right_split_tile(u0, tw), b = right_split_tile(u1, tw);
            const long long w = (long long)(b - a) * 4 - 2LL * std::max(0, std::min(b, tw) - std::min(a, tw));
            if (w > umax) umax = w;
        }
        const long long cost = waves * (umax + ovh);
        if (best_cost < 0 || cost < best_cost) {
            best_cost = cost;
            best = ns;
        }
    }
    return best;
}

// 2-D tensor map of a column-major ldw x K operand panel (V or Y; element (row, col) at
// base[row + col * ldw]) with a box of `rows` x K elements: one TMA copy moves rows r .. r+rows-1 of
// all K columns into a [col][rows] shared-memory tile (rows = SK: the padded, conflict-free stride);
// rows past ldw are zero-filled.  The driver entry point is resolved once through the runtime.
int ft_panel_tmap(CUtensorMap *m, const double *base, int64_t ldw, int K, int rows) {
    static PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    if (!enc) {
        void *fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess || !fn)
            return 1;
        enc = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
    }
    if (!base || K <= 0 || K > FT_NBMAX || (ldw * 8) % 16 != 0 || (((uintptr_t)base) & 15)) return 1;
    const cuuint64_t dims[2] = {(cuuint64_t)ldw, (cuuint64_t)K};
    const cuuint64_t strides[1] = {(cuuint64_t)ldw * sizeof(double)};
    const cuuint32_t box[2] = {(cuuint32_t)rows, (cuuint32_t)K};
    const cuuint32_t estr[2] = {1, 1};
    const CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<double *>(base), dims, strides, box, estr,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? 0 : 1;
}

// dynamic shared memory rounded up to a 128-byte boundary (TMA destinations); the offset is added
// to the shared array itself, so the compiler keeps the shared address space (LDS, not generic LD)
__device__ __forceinline__ unsigned char *align128(unsigned char *p) {
    return p + ((128u - (smem_u32(p) & 127u)) & 127u);
}

extern "C" int ft_debug_right_splits(int r_lo, int r_hi, int c_lo, int c_hi, int nsm, int extra_strips, int wr_lo) {
    return ft_gemm_splits(r_lo, r_hi, c_lo, c_hi, nsm, extra_strips, wr_lo);
}
extern "C" void ft_debug_right_split_range(int nrt, int tw, int ns, int y, int *t0, int *t1) {
    const long long units = (long long)tw + 2LL * (nrt - tw);
    if (t0) *t0 = right_split_tile((long long)y * units / ns, tw);
    if (t1) *t1 = right_split_tile((long long)(y + 1) * units / ns, tw);
}

template <int KT>
struct RightSmemT {
    double Vc[KT][SK];     // sign * V(cols, k) as [k][col]   (A operand of the right update)
    double Ys[2][KT][SK];  // Y(rows, k) as [k][row], double-buffered TMA tiles (B operand of the right update)
    double Vr[2][KT][SK];  // V(rows, j) as [j][row], double-buffered TMA tiles (B operand of W^T = C_new^T V)
    double Yn[KT];         // fold_row: Y(n, :) = Y_chk
};

// k-major operand tile: M(r .. r+63, 0:KT) (column-major, leading dim ld) -> T[k][row];
// rows >= hi and k >= K are zero-filled
template <int KT>
__device__ __forceinline__ void issue_ktile(double (*T)[SK], const double *M, int64_t ld, int r, int hi, int K) {
    for (int q = threadIdx.x; q < KT * (UB / 2); q += UT) {
        const int kk = q / (UB / 2), m2 = (q % (UB / 2)) * 2;
        const int left = hi - (r + m2);
        const int bytes = kk < K ? (left >= 2 ? 16 : (left == 1 ? 8 : 0)) : 0;
        cp_async16(&T[kk][m2], bytes ? M + (int64_t)kk * ld + r + m2 : M, bytes);
    }
}

// acc(pair) <- C(row, row+1 ; col) with rows outside [lo, hi) (or a missing column) as 0
__device__ __forceinline__ double2 load_pair(const double *colp, int row, int lo, int hi, bool colok) {
    double2 v = make_double2(0.0, 0.0);
    if (!colok) return v;
    if (row >= lo && row + 1 < hi) return *reinterpret_cast<const double2 *>(colp + row);
    if (row >= lo && row < hi) v.x = colp[row];
    if (row + 1 >= lo && row + 1 < hi) v.y = colp[row + 1];
    return v;
}
__device__ __forceinline__ void store_pair(double *colp, int row, int lo, int hi, bool colok, double x, double y) {
    if (!colok) return;
    if (row >= lo && row + 1 < hi) {
        *reinterpret_cast<double2 *>(colp + row) = make_double2(x, y);
        return;
    }
    if (row >= lo && row < hi) colp[row] = x;
    if (row + 1 >= lo && row + 1 < hi) colp[row + 1] = y;
}

// ---------------------------------------------------------------------------
// Right update A(rows, cols) += sign * Y V(cols,:)^T, fused W = V(wrows,:)^T A_new
// warp w owns columns w*8 .. w*8+7 of the strip and all 64 rows of a tile (8 fragments)
// ---------------------------------------------------------------------------
// the fused pre-update check (R15), evaluated redundantly by warp 0 of every CTA on the same
// inputs (so every CTA takes the same decision); returns the reason bits
__device__ int pre_update_reason(const GemmRightParams &p) {
    const FtCtl *ctl = p.pre_ctl;
    const int lane = threadIdx.x & 31, n = p.pre_n, ib = p.K;
    const double eps = 2.220446049250313e-16;
    const double unit = (double)n * eps * ctl->normF;
    const double tmax = __ldcg(&ctl->tmax);
    const double tauY = ctl->c_thr * unit * (tmax > 1.0 ? tmax : 1.0);
    const double tauV = ctl->c_thr * (double)n * eps * sqrt((double)n);
    int reason = __ldcg(&ctl->nflag) > 0 ? 1 : 0;
    for (int j = lane; j < ib; j += 32) {
        const double dy = __ldcg(&ctl->eY[j * FT_ESTR]) - __ldcg(p.Y + n + (int64_t)j * p.ldw);
        const double dv = __ldcg(&ctl->eV[j * FT_ESTR]) - __ldcg(p.V + n + (int64_t)j * p.ldw);
        if (not_within(dy, tauY)) reason |= 2;
        if (not_within(dv, tauV)) reason |= 4;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) reason |= __shfl_xor_sync(0xffffffffu, reason, o);
    return reason;
}

template <int KT>
__global__ void __launch_bounds__(UT, 1)
    k_gemm_right(const GemmRightParams p, const __grid_constant__ CUtensorMap tmY, const __grid_constant__ CUtensorMap tmV) {
    // the halt flag is loaded here but first used at the first tile's barrier (before any store),
    // so its round trip overlaps the operand loads instead of delaying them
    const int halted = p.ctl ? __ldcg(&p.ctl->halt) : 0;
    // the panel's T row sums for the T check of the strip's last CTA (which CTA is last is known
    // only at the end: every CTA prefetches, so the check carries no load round trip)
    const double tchk_pre = (p.tctl && p.Wt && (threadIdx.x & 3) == 0 && (int)(threadIdx.x >> 2) < p.K)
                                ? __ldcg(&p.tctl->tchk[threadIdx.x >> 2]) : 0.0;
    // fused pre-update check: warp 0 evaluates it while the other warps start the operand and
    // C-tile loads; the decision is read at the first tile's barrier, before any store
    __shared__ int s_reason;
    if (p.pre_ctl && threadIdx.x < 32) {
        const int reason = pre_update_reason(p);
        if (threadIdx.x == 0) s_reason = reason;
    }
    extern __shared__ unsigned char smem_raw[];
    RightSmemT<KT> &S = *reinterpret_cast<RightSmemT<KT> *>(align128(smem_raw));
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int lr = lane >> 2, lc = lane & 3;
    // the last strip of the grid is the M-part when present (rows 0..m_r_hi, no W)
    const bool mpart = p.has_m && blockIdx.x == gridDim.x - 1;
    const int r_lo = mpart ? 0 : p.r_lo, r_hi = mpart ? p.m_r_hi : p.r_hi;
    const int do_w = mpart ? 0 : p.do_w;
    const int cb = mpart ? p.m_c_lo : p.c_lo + blockIdx.x * UB;
    const int ncols = min(UB, (mpart ? p.m_c_hi : p.c_hi) - cb);
    const int K = p.K;
    const double sg = p.sign;
    const int rbase = (r_lo / UB) * UB;
    const int nrt = (r_hi - rbase + UB - 1) / UB;
    // this split's tiles: equal weights per split (right-only tiles 1, right + W tiles 2)
    const int tw = do_w ? (p.wr_lo <= rbase ? 0 : min(nrt, (p.wr_lo - rbase) / UB)) : nrt;
    const long long units = (long long)tw + 2LL * (nrt - tw);
    const int t0 = right_split_tile((long long)blockIdx.y * units / gridDim.y, tw);
    const int t1 = right_split_tile((long long)(blockIdx.y + 1) * units / gridDim.y, tw);
    constexpr int NJ = KT / 8;
    // fold_row: row p.r_hi (= n, the column checksum c) is updated by the last row split as a GEMV,
    // 4 lanes per strip column; c(col) is prefetched here, its use is after the tile loop
    const bool foldr = p.fold_row && !mpart && (int)blockIdx.y == (int)gridDim.y - 1;
    const int fcol = tid >> 2, fq = tid & 3;
    const double cold = (foldr && fq == 0 && fcol < ncols) ? __ldcg(p.A + p.r_hi + (int64_t)(cb + fcol) * p.lda) : 0.0;
    // warp tile: 16 columns x 32 rows (warp (wc, wr): columns wc*16.., rows wr*32.. of each tile):
    // per k step 2 + 4 fragment loads feed 8 DMMA (the W pass: 4 shuffles + 8 loads feed 16)
    const int wc = warp & 3, wr = warp >> 2;
    int cols2[2];
    bool colok2[2];
    double *colp2[2];
#pragma unroll
    for (int mi = 0; mi < 2; mi++) {
        cols2[mi] = wc * 16 + mi * 8 + lr;
        colok2[mi] = cols2[mi] < ncols;
        colp2[mi] = p.A + (int64_t)(cb + (colok2[mi] ? cols2[mi] : 0)) * p.lda;
    }

    // Operand pipeline: the Y / V row tiles (rows r .. r+SK-1, columns 0..K-1) arrive by 2-D tensor
    // TMA, one instruction per tile issued by thread 0, into double buffers; full[b] completes on the
    // copy's transaction count, empty[b] when all eight warps have read the buffer (mbarrier arrive:
    // no CTA-wide barrier inside the tile loop, so warps drift and the DMMA pipe stays fed while one
    // warp stores or shuffles).  Ys columns k >= K meet zero Vc entries: they start as zeros (stale
    // shared memory could hold NaN patterns); rows past the matrix are zero-filled by the TMA unit.
    __shared__ __align__(8) unsigned long long yfull[2], vfull[2], yempty[2], vempty[2];
    if (tid == 0) {
        for (int b = 0; b < 2; b++) {
            mbar_init(&yfull[b], 1);
            mbar_init(&vfull[b], 1);
            mbar_init(&yempty[b], UT / 32);
            mbar_init(&vempty[b], UT / 32);
        }
        mbar_fence_init();
        if (p.do_right) tma_prefetch_map(&tmY);
        if (do_w) tma_prefetch_map(&tmV);
    }
    const unsigned tile_bytes = (unsigned)(SK * K * 8);
    auto issue_y = [&](int tt, int b) {  // thread 0: tile tt's Y rows into buffer b
        mbar_expect_tx(&yfull[b], tile_bytes);
        tma_load_2d(&S.Ys[b][0][0], &tmY, rbase + tt * UB, 0, &yfull[b]);
    };
    auto issue_v = [&](int tt, int b) {  // thread 0: tile tt's V rows into buffer b
        mbar_expect_tx(&vfull[b], tile_bytes);
        tma_load_2d(&S.Vr[b][0][0], &tmV, rbase + tt * UB, 0, &vfull[b]);
    };
    if (K < KT && p.do_right)
        for (int i = tid; i < 2 * (KT - K) * SK; i += UT) {
            const int b = i / ((KT - K) * SK), rem = i % ((KT - K) * SK);
            S.Ys[b][K + rem / SK][rem % SK] = 0.0;
        }
    if (foldr && tid < KT) S.Yn[tid] = tid < K ? __ldcg(p.Y + p.r_hi + (int64_t)tid * p.ldw) : 0.0;
    __syncthreads();  // barrier init visible before the first copies
    // tiles above the W rows (tt < tw) run the right pass only: no V tile, no W pass (their W rows
    // are all masked); the V pipeline runs over this CTA's W tiles tv0 .. t1-1
    const int tv0 = max(t0, tw);
    const int ny_issued = (p.do_right && t0 < t1) ? min(2, t1 - t0) : 0;
    const int nv_issued = (do_w && tv0 < t1) ? min(2, t1 - tv0) : 0;
    if (tid == 0) {
        for (int b = 0; b < ny_issued; b++) issue_y(t0 + b, b);
        for (int b = 0; b < nv_issued; b++) issue_v(tv0 + b, b);
    }
    // sign * V(cols, :) once per CTA (sign folded into the A operand: the accumulators start from C
    // itself and hold C_new at the end -- the same roundings as sign * (sign C + V Y^T))
    if (p.do_right) {
        constexpr int NV = KT * UB / UT;
        double vv[NV];
#pragma unroll
        for (int m = 0; m < NV; m++) {
            const int i = tid + m * UT, kk = i / UB, cc = i % UB;
            const bool ok = kk < K && cc < ncols;
            const int vrow = ft_cmap(cb + cc, p.cm_G, p.cm_rank, p.cm_nb, p.cm_ncl, p.cm_n);
            vv[m] = ok ? __ldg(p.V + vrow + (int64_t)kk * p.ldw) : 0.0;
        }
#pragma unroll
        for (int m = 0; m < NV; m++) {
            const int i = tid + m * UT;
            S.Vc[i / UB][i % UB] = sg * vv[m];
        }
    }
    double wacc[2][NJ][2];
#pragma unroll
    for (int mi = 0; mi < 2; mi++)
#pragma unroll
        for (int a = 0; a < NJ; a++) wacc[mi][a][0] = wacc[mi][a][1] = 0.0;
    auto pre_abort = [&]() -> bool {  // after a __syncthreads that follows the evaluation
        const bool raise = !halted && p.pre_ctl && s_reason;
        if (!halted && !raise) return false;
        if (raise && threadIdx.x == 0 && blockIdx.x == 0 && blockIdx.y == 0) {
            FtCtl *ctl = p.pre_ctl;
            ctl->halt_panel = p.pre_panel;
            ctl->halt_stage = 1;
            ctl->halt_reason = s_reason;
            __threadfence();
            ctl->halt = 1;
        }
        // the copies in flight land before the CTA's shared memory is released
        for (int b = 0; b < ny_issued; b++) mbar_wait(&yfull[b], 0u);
        for (int b = 0; b < nv_issued; b++) mbar_wait(&vfull[b], 0u);
        return true;  // nothing consumed: the panel is redone from its checkpoint
    };
    // C tile of tile tt into registers (16-byte loads; masked pairs at the edges)
    auto load_c = [&](int tt, double2 (&dst)[2][4]) {
        const int r = rbase + tt * UB;
        const int lo = max(r, r_lo), hi = min(r + UB, r_hi);
        const bool full = lo == r && hi == r + UB && ncols == UB;
#pragma unroll
        for (int mi = 0; mi < 2; mi++)
#pragma unroll
            for (int ni = 0; ni < 4; ni++) {
                const int row = r + wr * 32 + ni * 8 + 2 * lc;
                dst[mi][ni] = full ? *reinterpret_cast<const double2 *>(colp2[mi] + row)
                                   : load_pair(colp2[mi], row, lo, hi, colok2[mi]);
            }
    };
    double2 cn[2][4];  // the next tile's C, prefetched a whole tile ahead
    if (t0 < t1) load_c(t0, cn);
    for (int tt = t0; tt < t1; tt++) {
        const int it = tt - t0, b = it & 1;
        const unsigned ph = (unsigned)(it >> 1) & 1u;
        const int r = rbase + tt * UB;
        const int lo = max(r, r_lo), hi = min(r + UB, r_hi);
        const bool full = lo == r && hi == r + UB && ncols == UB;  // interior tile: no masks
        double acc[2][4][2];
#pragma unroll
        for (int mi = 0; mi < 2; mi++)
#pragma unroll
            for (int ni = 0; ni < 4; ni++) {
                acc[mi][ni][0] = cn[mi][ni].x;
                acc[mi][ni][1] = cn[mi][ni].y;
            }
        if (tt + 1 < t1) load_c(tt + 1, cn);
        if (tt == t0) {
            __syncthreads();  // Vc and the pre-update decision
            if (pre_abort()) return;
        } else if (tid == 0 && tt + 1 < t1 && p.do_right) {
            // refill tile tt-1's Y buffer with tile tt+1 once every warp has released it (its right
            // pass: long done); the V buffer follows after this warp's own right pass, below
            mbar_wait(&yempty[b ^ 1], (unsigned)((it - 1) >> 1) & 1u);
            issue_y(tt + 1, b ^ 1);
        }
        if (p.do_right) {
            mbar_wait(&yfull[b], ph);
#pragma unroll 4
            for (int k0 = 0; k0 < KT; k0 += 4) {
                double a[2], bb[4];
#pragma unroll
                for (int mi = 0; mi < 2; mi++) a[mi] = S.Vc[k0 + lc][wc * 16 + mi * 8 + lr];
#pragma unroll
                for (int ni = 0; ni < 4; ni++) bb[ni] = S.Ys[b][k0 + lc][wr * 32 + ni * 8 + lr];
#pragma unroll
                for (int mi = 0; mi < 2; mi++)
#pragma unroll
                    for (int ni = 0; ni < 4; ni++) dmma_8x8x4(acc[mi][ni][0], acc[mi][ni][1], a[mi], bb[ni]);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&yempty[b]);
#pragma unroll
            for (int mi = 0; mi < 2; mi++)
#pragma unroll
                for (int ni = 0; ni < 4; ni++) {
                    const int row = r + wr * 32 + ni * 8 + 2 * lc;
                    if (full) *reinterpret_cast<double2 *>(colp2[mi] + row) = make_double2(acc[mi][ni][0], acc[mi][ni][1]);
                    else store_pair(colp2[mi], row, lo, hi, colok2[mi], acc[mi][ni][0], acc[mi][ni][1]);
                }
        }
        if (do_w && tt >= tw) {
            const int jv = tt - tv0, bv = jv & 1;  // this tile's place in the V pipeline
            if (tid == 0 && jv > 0 && tt + 1 < t1) {
                // refill the V buffer of the previous W tile with tile tt+1: by now every warp is
                // normally past that W pass, so this wait rarely blocks (and never blocks the Y refill)
                mbar_wait(&vempty[bv ^ 1], (unsigned)((jv - 1) >> 1) & 1u);
                issue_v(tt + 1, bv ^ 1);
            }
            mbar_wait(&vfull[bv], (unsigned)(jv >> 1) & 1u);
            // only rows in [wr_lo, wr_hi) take part in W (a uniform test: interior tiles skip the masks)
            const int wlo = max(lo, p.wr_lo), whi = min(hi, p.wr_hi);
            if (!(wlo == r && whi == r + UB)) {
#pragma unroll
                for (int mi = 0; mi < 2; mi++)
#pragma unroll
                    for (int ni = 0; ni < 4; ni++) {
                        const int row = r + wr * 32 + ni * 8 + 2 * lc;
                        if (row < wlo || row >= whi) acc[mi][ni][0] = 0.0;
                        if (row + 1 < wlo || row + 1 >= whi) acc[mi][ni][1] = 0.0;
                    }
            }
            // W^T(cols, j) += C_new^T(cols, rows) V(rows, j) over this warp's 32 rows.  The rows are
            // taken in a permuted order so that every A fragment is an accumulator the lane already
            // holds (no shuffles): k-step (ni, e) gives lane (lr, lc) the row 8 ni + 2 lc + (e ^ lc/2),
            // i.e. acc[mi][ni][e ^ lc/2]; the matching B rows V(row, j) then hit every shared-memory
            // bank exactly twice per warp (stride SK = 4 mod 16), like the other fragment loads
            const int sw = lc >> 1;
#pragma unroll
            for (int ks = 0; ks < 8; ks++) {
                const int ni = ks >> 1, e = ks & 1;
                double a[2];
#pragma unroll
                for (int mi = 0; mi < 2; mi++) a[mi] = sw ? acc[mi][ni][e ^ 1] : acc[mi][ni][e];
                const int row = wr * 32 + ni * 8 + 2 * lc + (e ^ sw);
#pragma unroll
                for (int nj = 0; nj < NJ; nj++) {
                    const double vb = S.Vr[bv][nj * 8 + lr][row];
#pragma unroll
                    for (int mi = 0; mi < 2; mi++) dmma_8x8x4(wacc[mi][nj][0], wacc[mi][nj][1], a[mi], vb);
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&vempty[bv]);
        }
    }
    if (t0 >= t1) {  // no tile: take the pre-update decision here (no strip counter on a halt)
        __syncthreads();
        if (pre_abort()) return;
    }
    if (foldr) {  // c(cols) += Y(n, :) (sign V(cols, :))^T (Vc and Yn in shared memory)
        double s0 = 0.0, s1 = 0.0;
#pragma unroll
        for (int kk = fq; kk < KT; kk += 8) {
            s0 += S.Vc[kk][fcol] * S.Yn[kk];
            s1 += S.Vc[kk + 4][fcol] * S.Yn[kk + 4];
        }
        s0 += s1;
        s0 += __shfl_xor_sync(0xffffffffu, s0, 1);
        s0 += __shfl_xor_sync(0xffffffffu, s0, 2);
        if (fq == 0 && fcol < ncols) p.A[p.r_hi + (int64_t)(cb + fcol) * p.lda] = cold + s0;
    }
    if (do_w) {
        // deterministic partial of this row split: Wpart[split][col][j]; the two row warps of each
        // column group meet in shared memory first (wr = 1 stores, wr = 0 adds and writes out)
        double *Wp = p.Wpart + (int64_t)blockIdx.y * p.wsplit_stride;
        double *red = &S.Ys[0][0][0];  // [col][64] scratch: every copy into Ys has completed
        __syncthreads();
        if (wr == 1)
#pragma unroll
            for (int mi = 0; mi < 2; mi++)
#pragma unroll
                for (int nj = 0; nj < NJ; nj++)
#pragma unroll
                    for (int v = 0; v < 2; v++) red[cols2[mi] * FT_NBMAX + nj * 8 + 2 * lc + v] = wacc[mi][nj][v];
        __syncthreads();
        if (wr == 0)
#pragma unroll
            for (int mi = 0; mi < 2; mi++)
                if (colok2[mi])
#pragma unroll
                    for (int nj = 0; nj < NJ; nj++)
#pragma unroll
                        for (int v = 0; v < 2; v++) {
                            const int jj = nj * 8 + 2 * lc + v;
                            if (jj < K)
                                Wp[(int64_t)(cb + cols2[mi]) * FT_NBMAX + jj] =
                                    wacc[mi][nj][v] + red[cols2[mi] * FT_NBMAX + jj];
                        }
        if (p.Wt) {
            // the last CTA of the strip sums the partials (fixed order) and forms W' = op(T) W
            __shared__ int last;
            __syncthreads();
            if (tid == 0) last = atom_add_acqrel_s32(&p.strip_done[blockIdx.x], 1) == (int)gridDim.y - 1;
            __syncthreads();
            if (last) {
                double(*Ts)[SK] = S.Vc;  // reuse: T as Ts[a][b] (KT x KT)
                double(*Ws)[SK] = reinterpret_cast<double(*)[SK]>(&S.Ys[0][0][0]);  // W as Ws[col][b] (64 x KT): spans both Ys buffers
                for (int i = tid; i < KT * KT; i += UT) {  // the upper triangle of T; zeros below it
                    const int a = i % KT, b = i / KT;
                    const bool ok = a < K && b < K && a <= b;
                    cp_async8(&Ts[a][b], ok ? p.T + a + b * FT_NBMAX : p.T, ok ? 8 : 0);
                }
                cp_async_commit();
                // W = sum of the row-split partials (fixed order), all of this thread's elements
                // at once: their loads are in flight together (one round trip per 16)
                constexpr int NE = UB * KT / UT;  // elements per thread
                const int ns = (int)gridDim.y;
                double wv[NE];
#pragma unroll
                for (int m = 0; m < NE; m++) wv[m] = 0.0;
#pragma unroll 1
                for (int sp = 0; sp < ns; sp += 2) {
                    double v0[NE], v1[NE];
#pragma unroll
                    for (int m = 0; m < NE; m++) {
                        const int i = tid + m * UT, cc = i / KT, bb = i % KT;
                        const bool ok = cc < ncols && bb < K;
                        const double *src = p.Wpart + (int64_t)(cb + cc) * FT_NBMAX + bb + (int64_t)sp * p.wsplit_stride;
                        v0[m] = ok ? __ldcg(src) : 0.0;
                        v1[m] = (ok && sp + 1 < ns) ? __ldcg(src + p.wsplit_stride) : 0.0;
                    }
#pragma unroll
                    for (int m = 0; m < NE; m++) wv[m] += v0[m] + v1[m];
                }
#pragma unroll
                for (int m = 0; m < NE; m++) {
                    const int i = tid + m * UT;
                    Ws[i / KT][i % KT] = wv[m];
                }
                cp_async_wait<0>();
                __syncthreads();
                if (p.tctl) {
                    // T checksum (R15 extended to T): the T this CTA is about to consume against the
                    // row sums the panel stored with it; a mismatch flags the iteration (tbad) and the
                    // left-update launch raises the halt (the right update itself completes in full)
                    double ts, tsa;
                    t_row_checksum([&](int a, int bb) { return Ts[a][bb]; }, tid >> 2, tid & 3, K, ts, tsa);
                    const int a = tid >> 2;
                    if ((tid & 3) == 0 && a < K &&
                        not_within(ts - tchk_pre, (double)K * 2.220446049250313e-16 * tsa))
                        p.tctl->tbad = 1;
                }
                // W' = op(T) W as a 64 x KT x KT DMMA product, D(col, a) = sum_b W(col, b) B(b, a) with
                // B = T^T (transT: T(b, a), b <= a) or T (T(a, b), b >= a); the zeros below T's diagonal
                // restrict the sums.  Warp tile 16 x 32 as in the update (conflict-free fragments)
                {
                    const int wc = warp & 3, wr = warp >> 2;
                    double wacc2[2][4][2];
#pragma unroll
                    for (int mi = 0; mi < 2; mi++)
#pragma unroll
                        for (int ni = 0; ni < 4; ni++) wacc2[mi][ni][0] = wacc2[mi][ni][1] = 0.0;
                    if (KT == 64 ? wr * 32 < KT : true) {
                        if (p.transT)
                            warp_mma2<2, 4, false, true>(wacc2, &Ws[0][0], SK, &Ts[0][0], SK, wc * 16, wr * 32 % KT, KT);
                        else
                            warp_mma2<2, 4, false, false>(wacc2, &Ws[0][0], SK, &Ts[0][0], SK, wc * 16, wr * 32 % KT, KT);
                    }
#pragma unroll
                    for (int mi = 0; mi < 2; mi++)
#pragma unroll
                        for (int ni = 0; ni < 4; ni++)
#pragma unroll
                            for (int v = 0; v < 2; v++) {
                                const int cc = wc * 16 + mi * 8 + lr, a = (wr * 32 % KT) + ni * 8 + 2 * lc + v;
                                if (cc < ncols && a < K && (KT == 64 || wr == 0))
                                    p.Wt[(int64_t)(cb + cc) * FT_NBMAX + a] = wacc2[mi][ni][v];
                            }
                }
                if (tid == 0) p.strip_done[blockIdx.x] = 0;
            }
        }
    }
}

template <int KT>
static cudaError_t launch_right_kt(const GemmRightParams &p, cudaStream_t s) {
    static unsigned attr = 0;
    const unsigned dbit = ft_dev_bit();
    const size_t smem = sizeof(RightSmemT<KT>) + 128;  // + alignment slack (TMA destinations)
    if (!(attr & dbit)) {
        cudaError_t e = cudaFuncSetAttribute(k_gemm_right<KT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr |= dbit;
    }
    GemmRightParams q = p;
    q.fold_row = p.fold_row && p.do_right && p.cm_G <= 1 && p.r_hi - 1 > p.r_lo ? 1 : 0;
    if (q.fold_row) q.r_hi = p.r_hi - 1;  // row r_hi-1 (c) is folded into the last row split
    const int nstrip = (q.c_hi - q.c_lo + UB - 1) / UB + (q.has_m ? 1 : 0);
    const int ny = q.nsplit > 0 ? q.nsplit : 1;
    CUtensorMap tmY, tmV;
    memset(&tmY, 0, sizeof(tmY));
    memset(&tmV, 0, sizeof(tmV));
    if (q.do_right && ft_panel_tmap(&tmY, q.Y, q.ldw, q.K, SK)) return cudaErrorInvalidValue;
    if (q.do_w && ft_panel_tmap(&tmV, q.V, q.ldw, q.K, SK)) return cudaErrorInvalidValue;
    g_ft_launches++;
    k_gemm_right<KT><<<dim3(nstrip, ny), UT, smem, s>>>(q, tmY, tmV);
    return cudaGetLastError();
}
cudaError_t ft_launch_gemm_right(const GemmRightParams &p, cudaStream_t s) {
    if (p.K <= 0) return cudaSuccess;
    if (p.r_hi <= p.r_lo || p.c_hi <= p.c_lo) {  // no trailing block: at most the M-part
        if (!p.has_m || p.m_r_hi <= 0 || p.m_c_hi <= p.m_c_lo) return cudaSuccess;
        GemmRightParams q = p;
        q.has_m = 0;
        q.r_lo = 0;
        q.r_hi = p.m_r_hi;
        q.c_lo = p.m_c_lo;
        q.c_hi = p.m_c_hi;
        q.do_w = 0;
        q.Wt = nullptr;
        return ft_launch_gemm_right(q, s);
    }
    if (p.has_m && (p.m_r_hi <= 0 || p.m_c_hi <= p.m_c_lo)) {
        GemmRightParams q = p;
        q.has_m = 0;
        return ft_launch_gemm_right(q, s);
    }
    if (p.do_w && p.nsplit > FT_WSPLIT_MAX) return cudaErrorInvalidValue;
    const bool aligned = (p.lda % 2 == 0) && ((((uintptr_t)p.A) & 15) == 0) && (p.ldw % 2 == 0) &&
                         ((((uintptr_t)p.V) & 15) == 0) && (!p.do_right || ((((uintptr_t)p.Y) & 15) == 0));
    if (!aligned) return cudaErrorInvalidValue;  // the library only passes 16-byte aligned operands
    return p.K <= 32 ? launch_right_kt<32>(p, s) : launch_right_kt<64>(p, s);
}

// ---------------------------------------------------------------------------
// Left update: A(rows, cols) += sign * V(rows,:) (op(T) W(:, cols))
// warp (wc, wr) owns columns wc*16 .. +16 and rows wr*32 .. +32 of a 64 x 64 tile
// ---------------------------------------------------------------------------
template <int KT>
struct LeftSmemT {
    double Wc[UB][SK];     // sign * W' (W' = op(T) W) as [col][k]  (A operand, W'^T; stride SK: conflict free)
    double Vr[2][KT][SK];  // V(rows, k) as [k][row]    (B operand), double-buffered TMA tiles
    double Wr[KT];         // fold: W'(:, n), the r column's coefficients
    double Vn[KT];         // fold: V(n, :) = V_chk
};

// W'(col, a) = sum_b op(T)(a, b) W(b, col), W = sum over the row-split partials (fixed
// order); T upper triangular; W partials [split][col][64], W' [col][64]
__global__ void k_wprep(const double *__restrict__ Wpart, int64_t wstride, int nsplit,
                        const double *__restrict__ T, double *__restrict__ Wt, int c_lo, int c_hi, int K,
                        int transT, const FtCtl *ctl) {
    if (ctl && ctl->halt) return;
    __shared__ double Ts[FT_NBMAX][FT_NBMAX + 1];
    __shared__ double Ws[UT / FT_NBMAX][FT_NBMAX];
    for (int i = threadIdx.x; i < K * K; i += blockDim.x) {
        int a = i % K, b = i / K;
        Ts[a][b] = T[a + b * FT_NBMAX];
    }
    const int a = threadIdx.x % FT_NBMAX, cl = threadIdx.x / FT_NBMAX;
    const int col = c_lo + blockIdx.x * (blockDim.x / FT_NBMAX) + cl;
    double w = 0.0;
    if (col < c_hi && a < K) w = sum_strided(Wpart + (int64_t)col * FT_NBMAX + a, wstride, nsplit);
    Ws[cl][a] = w;
    __syncthreads();
    if (col >= c_hi || a >= K) return;
    double s0 = 0.0, s1 = 0.0;
    if (transT) {
        int b = 0;
        for (; b + 1 <= a; b += 2) {
            s0 += Ts[b][a] * Ws[cl][b];
            s1 += Ts[b + 1][a] * Ws[cl][b + 1];
        }
        if (b <= a) s0 += Ts[b][a] * Ws[cl][b];
    } else {
        int b = a;
        for (; b + 1 < K; b += 2) {
            s0 += Ts[a][b] * Ws[cl][b];
            s1 += Ts[a][b + 1] * Ws[cl][b + 1];
        }
        if (b < K) s0 += Ts[a][b] * Ws[cl][b];
    }
    Wt[(int64_t)col * FT_NBMAX + a] = s0 + s1;
}

template <int KT>
__global__ void __launch_bounds__(UT, 2) k_gemm_left(const GemmLeftParams p, const __grid_constant__ CUtensorMap tmV) {
    // both flags in flight together; they are first needed before this CTA's first global store,
    // so their round trip overlaps the CTA's first loads (the operand strip, the first tiles)
    const int halted = p.ctl ? __ldcg(&p.ctl->halt) : 0;
    const int tbad = p.tctl ? __ldcg(&p.tctl->tbad) : 0;
    // the right update consumed a corrupted T: nothing here runs, CTA (0, 0) raises the halt
    auto stop = [&]() -> bool {
        if (halted) return true;
        if (!tbad) return false;
        if (blockIdx.x == 0 && blockIdx.y == 0 && threadIdx.x == 0) {
            FtCtl *ctl = p.tctl;
            ctl->halt_panel = p.panel;
            ctl->halt_stage = 3;
            ctl->halt_reason = 32;
            __threadfence();
            ctl->halt = 1;
        }
        return true;
    };
    if ((int)blockIdx.y < p.nyf) {
        // frozen row sums of the panel columns k..e-1 (final now, untouched by this launch; R6):
        // Fr(i) += sum_{col in [max(k, i-1), e)} A(i, col) for i <= e -- one row per thread in
        // extra CTA rows of the grid, so the tile CTAs (few at late panels) carry no serial tail;
        // they come first in the grid (scheduled first, off the launch's tail)
        const int k = p.r_lo - 1, e = p.c_lo, rows = min(e + 1, p.n);
        const int i = (blockIdx.y * gridDim.x + blockIdx.x) * UT + threadIdx.x;
        if (i >= rows) {
            stop();
            return;
        }
        const double *a = p.A + i;
        // all of a row's loads in flight together (<= 64 columns): 8 at a time into 8 chains
        double s[8] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
        int c = max(k, i - 1);
#pragma unroll 8
        for (; c + 8 <= e; c += 8) {
#pragma unroll
            for (int u = 0; u < 8; u++) s[u] += __ldcg(a + (int64_t)(c + u) * p.lda);
        }
#pragma unroll
        for (int u = 0; u < 7; u++)
            if (c + u < e) s[u] += __ldcg(a + (int64_t)(c + u) * p.lda);
        if (stop()) return;
        p.Fr[i] += ((s[0] + s[1]) + (s[2] + s[3])) + ((s[4] + s[5]) + (s[6] + s[7]));
        return;
    }
    extern __shared__ unsigned char smem_raw[];
    LeftSmemT<KT> &S = *reinterpret_cast<LeftSmemT<KT> *>(align128(smem_raw));
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int lr = lane >> 2, lc = lane & 3;
    const int wc = warp & 3, wr = warp >> 2;
    // strips and row splits in reverse grid order: the CTAs of the last strip and the last row
    // split (the fold and the end-check tail) are scheduled first
    const int bx = (int)gridDim.x - 1 - (int)blockIdx.x, by = p.ny - 1 - ((int)blockIdx.y - p.nyf);
    const int cb = p.c_lo + bx * UB;
    const int ncols = min(UB, p.c_hi - cb);
    const int K = p.K;
    const double sg = p.sign;
    const int rbase = (p.r_lo / UB) * UB;
    const int nrt = (p.r_hi - rbase + UB - 1) / UB;
    const int t0 = (int)((long long)by * nrt / p.ny);
    const int t1 = (int)((long long)(by + 1) * nrt / p.ny);

    // V tiles (rows r .. r+SK-1, columns 0..K-1) by 2-D tensor TMA, one instruction per tile issued
    // by thread 0, into a double buffer: full[b] completes on the copy's transaction count, empty[b]
    // when all eight warps have read the buffer (no CTA-wide barrier inside the tile loop).  Columns
    // k >= K meet zero W' entries, so they are zeroed once (stale shared memory could hold NaN
    // patterns); rows past the matrix are zero-filled by the TMA unit.
    __shared__ __align__(8) unsigned long long vfull[2], vempty[2];
    if (tid == 0) {
        for (int b = 0; b < 2; b++) {
            mbar_init(&vfull[b], 1);
            mbar_init(&vempty[b], UT / 32);
        }
        mbar_fence_init();
        tma_prefetch_map(&tmV);
    }
    if (K < KT)
        for (int i = tid; i < 2 * (KT - K) * SK; i += UT) {
            const int b = i / ((KT - K) * SK), rem = i % ((KT - K) * SK);
            S.Vr[b][K + rem / SK][rem % SK] = 0.0;
        }
    // fold (ABFT): column n (r) rides with the last strip, row n (c) with the last row tile
    if (p.fold && tid < KT) {
        S.Wr[tid] = tid < K ? p.Wpart[(int64_t)p.n * FT_NBMAX + tid] : 0.0;
        S.Vn[tid] = tid < K ? p.V[p.n + (int64_t)tid * p.ldw] : 0.0;
    }
    __syncthreads();  // barrier init visible before the first copies
    const unsigned tile_bytes = (unsigned)(SK * K * 8);
    auto issue_v = [&](int tt, int b) {  // thread 0
        mbar_expect_tx(&vfull[b], tile_bytes);
        tma_load_2d(&S.Vr[b][0][0], &tmV, rbase + tt * UB, 0, &vfull[b]);
    };
    if (tid == 0 && t0 < t1) {
        issue_v(t0, 0);
        if (t0 + 1 < t1) issue_v(t0 + 1, 1);
    }
    // sign * W'^T for the strip: Wt [col][64] -> Wc[k][col] (sign folded into the A operand: the
    // accumulators start from C itself -- the same roundings as sign * (sign C + W'^T V^T))
    {
        constexpr int NW = KT * UB / UT;
        double wv[NW];
#pragma unroll
        for (int m = 0; m < NW; m++) {
            const int i = tid + m * UT, cc = i / KT, kk = i % KT;
            const bool ok = kk < K && cc < ncols;
            wv[m] = ok ? __ldcg(p.Wpart + (int64_t)(cb + cc) * FT_NBMAX + kk) : 0.0;
        }
#pragma unroll
        for (int m = 0; m < NW; m++) {
            const int i = tid + m * UT;
            S.Wc[i / KT][i % KT] = sg * wv[m];
        }
    }
    int cols[2];
    bool colok[2];
    double *colp[2];
#pragma unroll
    for (int mi = 0; mi < 2; mi++) {
        cols[mi] = wc * 16 + mi * 8 + lr;
        colok[mi] = cols[mi] < ncols;
        colp[mi] = p.A + (int64_t)(cb + (colok[mi] ? cols[mi] : 0)) * p.lda;
    }
    // fused end check: this CTA's share of sum r and sum c -- the entries it writes (column n:
    // r(k+1:n), row n: c(e:n)) in the tile epilogues, and a grid-strided slice of the entries
    // this launch does not touch (r(0:k+1), c(0:e), final since the right update / panel)
    // With the fold only the CTAs that write r or c (last strip, last tile row) take part:
    // the other CTAs skip the tail, so the serialised same-address atomics of the last-CTA
    // protocol scale with gx + gy instead of gx * gy (one CTA per tile at large n)
    double es_r = 0.0, es_c = 0.0;
    const int en = p.n;
    const bool fold_col = p.fold && bx == (int)gridDim.x - 1;
    const bool fold_row = p.fold && by == p.ny - 1;
    const bool part = !p.fold || fold_col || fold_row;
    const int pidx = !p.fold ? by * (int)gridDim.x + bx : (fold_col ? by : p.ny + bx);
    const int pcnt = !p.fold ? (int)gridDim.x * p.ny : (int)gridDim.x + p.ny - 1;
    if (p.endcheck && part) {
        const int nb = pcnt, b = pidx;
        const int nr = p.r_lo, ncc = p.c_lo;  // r(0:k+1), c(0:e)
        for (int x = b * UT + tid; x < nr + ncc; x += nb * UT) {
            if (x < nr) es_r += __ldcg(p.A + x + (int64_t)en * p.lda);
            else es_c += __ldcg(p.A + en + (int64_t)(x - nr) * p.lda);
        }
    }
    // C tile of tile tt into registers, prefetched a whole tile ahead (16-byte loads, masked edges)
    auto load_c = [&](int tt, double2 (&dst)[2][4]) {
        const int r = rbase + tt * UB;
        const int lo = max(r, p.r_lo), hi = min(r + UB, p.r_hi);
        const bool full = lo == r && hi == r + UB && ncols == UB;
#pragma unroll
        for (int mi = 0; mi < 2; mi++)
#pragma unroll
            for (int ni = 0; ni < 4; ni++) {
                const int row = r + wr * 32 + ni * 8 + 2 * lc;
                dst[mi][ni] = full ? *reinterpret_cast<const double2 *>(colp[mi] + row)
                                   : load_pair(colp[mi], row, lo, hi, colok[mi]);
            }
    };
    double2 cn[2][4];
    if (t0 < t1) load_c(t0, cn);
    if (stop()) {  // before any global store; the copies in flight land before the CTA exits
        for (int b = 0; b < 2 && t0 + b < t1; b++) mbar_wait(&vfull[b], 0u);
        return;
    }
    if (p.pre_reset && bx == 0 && by == 0) {  // the right update has read them
        for (int j = tid; j < FT_NBMAX; j += UT) {
            p.pre_reset->eY[j * FT_ESTR] = 0.0;
            p.pre_reset->eV[j * FT_ESTR] = 0.0;
        }
        if (tid == 0) p.pre_reset->nflag = 0;
    }
    __syncthreads();  // every thread's part of sign * W' landed
    for (int tt = t0; tt < t1; tt++) {
        const int it = tt - t0, st = it & 1;
        const int r = rbase + tt * UB;
        const int lo = max(r, p.r_lo), hi = min(r + UB, p.r_hi);
        const bool full = lo == r && hi == r + UB && ncols == UB;  // interior tile: no masks
        double acc[2][4][2];
#pragma unroll
        for (int mi = 0; mi < 2; mi++)
#pragma unroll
            for (int ni = 0; ni < 4; ni++) {
                acc[mi][ni][0] = cn[mi][ni].x;
                acc[mi][ni][1] = cn[mi][ni].y;
            }
        if (tt + 1 < t1) {
            load_c(tt + 1, cn);
            if (tid == 0 && it >= 1) {  // refill tile tt-1's buffer with tile tt+1 once every warp released it
                mbar_wait(&vempty[st ^ 1], (unsigned)((it - 1) >> 1) & 1u);
                issue_v(tt + 1, st ^ 1);
            }
        }
        mbar_wait(&vfull[st], (unsigned)(it >> 1) & 1u);
#pragma unroll 4
        for (int k0 = 0; k0 < KT; k0 += 4) {
            double a[2], b[4];
#pragma unroll
            for (int mi = 0; mi < 2; mi++) a[mi] = S.Wc[wc * 16 + mi * 8 + lr][k0 + lc];
#pragma unroll
            for (int ni = 0; ni < 4; ni++) b[ni] = S.Vr[st][k0 + lc][wr * 32 + ni * 8 + lr];
#pragma unroll
            for (int mi = 0; mi < 2; mi++)
#pragma unroll
                for (int ni = 0; ni < 4; ni++) dmma_8x8x4(acc[mi][ni][0], acc[mi][ni][1], a[mi], b[ni]);
        }
        if (fold_col) {  // r(rows) += sg V(rows, :) W'(:, n): 4 lanes per row, two chains each
            const int rr = tid >> 2, q4 = tid & 3;
            double s0 = 0.0, s1 = 0.0;
#pragma unroll
            for (int kk = q4; kk < KT; kk += 8) {
                s0 += S.Vr[st][kk][rr] * S.Wr[kk];
                s1 += S.Vr[st][kk + 4][rr] * S.Wr[kk + 4];
            }
            s0 += s1;
            s0 += __shfl_xor_sync(0xffffffffu, s0, 1);
            s0 += __shfl_xor_sync(0xffffffffu, s0, 2);
            const int row = r + rr;
            if (q4 == 0 && row >= lo && row < hi) {
                double *pr = p.A + row + (int64_t)p.n * p.lda;
                const double v = *pr + sg * s0;
                *pr = v;
                es_r += v;
            }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&vempty[st]);  // this warp is done with Vr[st]
#pragma unroll
        for (int mi = 0; mi < 2; mi++)
#pragma unroll
            for (int ni = 0; ni < 4; ni++) {
                const int row = r + wr * 32 + ni * 8 + 2 * lc;
                const double x = acc[mi][ni][0], y = acc[mi][ni][1];
                if (full) *reinterpret_cast<double2 *>(colp[mi] + row) = make_double2(x, y);
                else store_pair(colp[mi], row, lo, hi, colok[mi], x, y);
                if (p.endcheck && !p.fold && colok[mi]) {  // fold: r, c are written by the fold code
                    const int gc = cb + cols[mi];
                    const bool in0 = row >= lo && row < hi, in1 = row + 1 >= lo && row + 1 < hi;
                    if (gc == en) {  // r entries (kappa = row n excluded)
                        if (in0 && row < en) es_r += x;
                        if (in1 && row + 1 < en) es_r += y;
                    } else if (gc < en) {  // c entries
                        if (in0 && row == en) es_c += x;
                        if (in1 && row + 1 == en) es_c += y;
                    }
                }
            }
    }
    if (fold_row) {  // c(cols) += sg V(n, :) W'(:, cols), and kappa with the last strip
        __syncthreads();
        const int cc = tid >> 2, q4 = tid & 3;
        double s0 = 0.0, s1 = 0.0, k0 = 0.0, k1 = 0.0;
#pragma unroll
        for (int kk = q4; kk < KT; kk += 8) {
            s0 += S.Vn[kk] * S.Wc[cc][kk];  // Wc = sign * W': the sign is in s0
            s1 += S.Vn[kk + 4] * S.Wc[cc][kk + 4];
            k0 += S.Vn[kk] * S.Wr[kk];
            k1 += S.Vn[kk + 4] * S.Wr[kk + 4];
        }
        s0 += s1;
        s0 += __shfl_xor_sync(0xffffffffu, s0, 1);
        s0 += __shfl_xor_sync(0xffffffffu, s0, 2);
        k0 += k1;
        k0 += __shfl_xor_sync(0xffffffffu, k0, 1);
        k0 += __shfl_xor_sync(0xffffffffu, k0, 2);
        if (q4 == 0 && cc < ncols) {
            double *pc = p.A + p.n + (int64_t)(cb + cc) * p.lda;
            const double v = *pc + s0;
            *pc = v;
            es_c += v;
        }
        if (fold_col && tid == 0) {
            double *pk = p.A + p.n + (int64_t)p.n * p.lda;
            *pk = *pk + sg * k0;
        }
    }
    if (!p.endcheck || !part) return;  // (the fold's stores reach the last CTA through the acq_rel below)
    // fused end-of-iteration check (Alg. 3 l.12-13; R11/R22): the CTA's partial sums go into
    // ctl->sums[2:4]; once every CTA has finished, the last one compares sum r and sum c with
    // kappa (EAGER) or with each other (PAPER)
    __shared__ int last;
    __shared__ double red2[2][UT / 32];
    es_r = warp_sum(es_r);
    es_c = warp_sum(es_c);
    if (lane == 0) {
        red2[0][warp] = es_r;
        red2[1][warp] = es_c;
    }
    __syncthreads();
    if (tid == 0) {
        double a = 0.0, b = 0.0;
        for (int w = 0; w < UT / 32; w++) {
            a += red2[0][w];
            b += red2[1][w];
        }
        atomicAdd(&p.ectl->sums[2], a);
        atomicAdd(&p.ectl->sums[3], b);
        // deferred: the next panel launch compares the sums (kernel boundary orders them)
        last = p.endcheck == 2 ? 0 : atom_add_acqrel_s32(&p.ectl->done_left, 1) == pcnt - 1;
    }
    __syncthreads();
    if (!last || tid != 0) return;
    const int n = p.n;
    const double Sr = __ldcg(&p.ectl->sums[2]), Sc = __ldcg(&p.ectl->sums[3]);
    p.ectl->sums[2] = 0.0;
    p.ectl->sums[3] = 0.0;
    FtCtl *ctl = p.ectl;
    const double kap = __ldcg(p.A + n + (int64_t)n * p.lda);
    const double tauS = ctl->c_thr * (double)n * 2.220446049250313e-16 * ctl->normF * sqrt((double)n);
    int reason = 0;
    if (p.policy == FT_POLICY_PAPER) {
        if (not_within(Sr - Sc, tauS)) reason |= 8;
    } else {
        if (not_within(Sr - kap, tauS) || not_within(Sc - kap, tauS)) reason |= 8;
    }
    ctl->done_left = 0;
    if (reason) {
        ctl->halt_panel = p.panel;
        ctl->halt_stage = 2;
        ctl->halt_reason = reason;
        __threadfence();
        ctl->halt = 1;
    }
}

template <int KT>
static cudaError_t launch_left_kt(const GemmLeftParams &p, cudaStream_t s) {
    static unsigned attr = 0;
    const unsigned dbit = ft_dev_bit();
    const size_t smem = sizeof(LeftSmemT<KT>) + 128;  // + alignment slack (TMA destinations)
    if (!(attr & dbit)) {
        cudaError_t e = cudaFuncSetAttribute(k_gemm_left<KT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr |= dbit;
    }
    // fold: tiles cover rows [r_lo, r_hi-1) and columns [c_lo, c_hi-1); the checksum row and
    // column (index n) are folded into the last tile row / strip
    const bool fold = p.fold && p.r_hi - 1 == p.n && p.c_hi - 1 == p.n && p.r_hi - 1 > p.r_lo &&
                      p.c_hi - 1 > p.c_lo && p.wt_ready;
    const int r_hi = fold ? p.r_hi - 1 : p.r_hi, c_hi = fold ? p.c_hi - 1 : p.c_hi;
    const int nstrip = (c_hi - p.c_lo + UB - 1) / UB;
    static int nsm = 0;
    if (!nsm) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    }
    const int nrt = (r_hi - (p.r_lo / UB) * UB + UB - 1) / UB;
    // per-CTA prologue of half a tile (W' strip + first V tile): measured best of 0 / 2 / 4 / 8 at
    // n = 8192 / 16384 (profiles/r01/s8/left_ovh.txt); FT_LEFT_OVH overrides for sweeps
    static const int ovh = getenv("FT_LEFT_OVH") ? atoi(getenv("FT_LEFT_OVH")) : 2;
    const int ny = best_splits(nstrip, nrt, nsm, 1 << 20, 2, ovh);  // two resident CTAs per SM
    if (!p.wt_ready) {
        g_ft_launches++;
        const int per = UT / FT_NBMAX;  // columns per k_wprep block
        k_wprep<<<(p.c_hi - p.c_lo + per - 1) / per, UT, 0, s>>>(p.Wpart, p.wsplit_stride,
                                                                  p.nsplit > 0 ? p.nsplit : 1, p.T, p.Wt, p.c_lo,
                                                                  p.c_hi, p.K, p.transT, p.ctl);
    }
    g_ft_launches++;
    GemmLeftParams q = p;
    q.Wpart = p.Wt;  // the main kernel reads W' = op(T) W
    q.fold = fold ? 1 : 0;
    q.r_hi = r_hi;
    q.c_hi = c_hi;
    q.ny = ny;
    int nyf = 0;  // extra CTA rows for the frozen row sums (one row of A per thread)
    if (p.endcheck && p.Fr) {
        const int rows = std::min(p.c_lo + 1, p.n);
        nyf = ((rows + UT - 1) / UT + nstrip - 1) / nstrip;
    }
    q.nyf = nyf;
    CUtensorMap tmV;
    memset(&tmV, 0, sizeof(tmV));
    if (ft_panel_tmap(&tmV, q.V, q.ldw, q.K, SK)) return cudaErrorInvalidValue;
    k_gemm_left<KT><<<dim3(nstrip, ny + nyf), UT, smem, s>>>(q, tmV);
    return cudaGetLastError();
}
cudaError_t ft_launch_gemm_left(const GemmLeftParams &p, cudaStream_t s) {
    if (p.r_hi <= p.r_lo || p.c_hi <= p.c_lo || p.K <= 0) return cudaSuccess;
    const bool aligned = (p.lda % 2 == 0) && ((((uintptr_t)p.A) & 15) == 0) && (p.ldw % 2 == 0) &&
                         ((((uintptr_t)p.V) & 15) == 0);
    if (!aligned) return cudaErrorInvalidValue;
    return p.K <= 32 ? launch_left_kt<32>(p, s) : launch_left_kt<64>(p, s);
}

// ---------------------------------------------------------------------------
// Y_top (DLAHR2's final step): Y(0:k+1, :) = A(0:k+1, k+1:ihi) V(k+1:ihi, :) T,
// split over the long inner dimension; the same pass sums A's rows for the
// verify-before-consume check of the rows above the panel (area 1).
// ---------------------------------------------------------------------------
#ifndef YT_M
#define YT_M 64  // rows per CTA (16 per warp)
#endif
#define YT_T (2 * YT_M)  // threads per CTA
#define YT_K 32
struct YtopSmem {
    double As[2][YT_K * (YT_M + 4)];      // A tile [col][row], double-buffered
    double Vs[2][FT_NBMAX * (YT_K + 4)];  // V [j][col]
};

__global__ void __launch_bounds__(YT_T) k_ytop_partial(YtopParams p) {
    if (p.ctl->halt) return;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    YtopSmem &S = *reinterpret_cast<YtopSmem *>(smem_raw);
    const int warp = threadIdx.x >> 5;
    const int m_lo = blockIdx.x * YT_M;
    const int mrows = min(YT_M, p.k + 1 - m_lo);
    const bool mg = p.cm_G > 1;
    const int K0 = mg ? p.kc0 : p.k + 1, K1 = mg ? p.kc1 : p.ihi;  // inner range (local columns)
    const int nkt = (K1 - K0 + YT_K - 1) / YT_K;
    const int kt0 = (int)((long long)blockIdx.y * nkt / gridDim.y);
    const int kt1 = (int)((long long)(blockIdx.y + 1) * nkt / gridDim.y);
    const int ib = p.ib;
    double acc[2][8][2];
#pragma unroll
    for (int a = 0; a < 2; a++)
#pragma unroll
        for (int b = 0; b < 8; b++) acc[a][b][0] = acc[a][b][1] = 0.0;
    double rs = 0.0;
    // stage k-tile kt into buffer st with cp.async (every load in flight at once)
    auto issue = [&](int kt, int st) {
        const int kc = K0 + kt * YT_K;
        const int nk = min(YT_K, K1 - kc);
        for (int i = threadIdx.x; i < YT_K * (YT_M / 2); i += blockDim.x) {  // 16-byte row pairs
            const int m2 = (i % (YT_M / 2)) * 2, kk = i / (YT_M / 2);
            const int bytes = kk < nk ? (m2 + 1 < mrows ? 16 : (m2 < mrows ? 8 : 0)) : 0;
            cp_async16(&S.As[st][kk * (YT_M + 4) + m2], bytes ? p.A + (m_lo + m2) + (int64_t)(kc + kk) * p.ldw : p.A,
                       bytes);
        }
        for (int i = threadIdx.x; i < FT_NBMAX * YT_K; i += blockDim.x) {
            const int kk = i % YT_K, jj = i / YT_K;
            const bool ok = jj < ib && kk < nk;
            const int vrow = mg ? ft_cmap(kc + kk, p.cm_G, p.cm_rank, p.cm_nb, p.cm_ncl, -1) : kc + kk;
            cp_async8(&S.Vs[st][jj * (YT_K + 4) + kk], ok ? p.V + vrow + (int64_t)jj * p.ldw : p.V, ok ? 8 : 0);
        }
    };
    if (kt0 < kt1) issue(kt0, 0);
    cp_async_commit();
    for (int kt = kt0; kt < kt1; kt++) {
        const int st = (kt - kt0) & 1;
        const int nk = min(YT_K, K1 - (K0 + kt * YT_K));
        if (kt + 1 < kt1) issue(kt + 1, st ^ 1);
        cp_async_commit();
        cp_async_wait<1>();
        __syncthreads();
        if (p.verify)  // row sums: row threadIdx.x % 64, alternate k of the tile per half of the CTA
            for (int kk = threadIdx.x / YT_M; kk < nk; kk += 2) rs += S.As[st][kk * (YT_M + 4) + (threadIdx.x % YT_M)];
        // warp tile: rows warp*16..+16, cols 0..63 (MI=2, NI=8)
        warp_mma<2, 8, true>(acc, S.As[st], YT_M + 4, S.Vs[st], YT_K + 4, warp * 16, 0, YT_K);
        __syncthreads();  // buffer st is refilled by the next iteration's issue
    }
    cp_async_wait<0>();
    double *yp = p.ypart + (int64_t)blockIdx.y * (int64_t)(p.k + 1) * FT_NBMAX;
#pragma unroll
    for (int mi = 0; mi < 2; mi++)
#pragma unroll
        for (int ni = 0; ni < 8; ni++)
#pragma unroll
            for (int v = 0; v < 2; v++) {
                int m = warp * 16 + frag_row(mi), jj = frag_col(ni, v);
                if (m < mrows && jj < ib) yp[(int64_t)(m_lo + m) * FT_NBMAX + jj] = acc[mi][ni][v];
            }
    if (p.verify) {  // the two halves' row sums meet in shared memory (the A tiles are free now)
        __syncthreads();
        double *half = &S.As[0][0];
        if (threadIdx.x >= YT_M) half[threadIdx.x - YT_M] = rs;
        __syncthreads();
        if (threadIdx.x < mrows) p.rowpart[(int64_t)blockIdx.y * (p.k + 1) + m_lo + threadIdx.x] = rs + half[threadIdx.x];
    }
}

// Y_top rows: sum the split partials, multiply by T; row-sum verify of area 1.
// Block = 16 rows x 64 columns of Y.
#define YF_R 16  // rows per row group (a thread per (row, j) of the group)
#define YF_G 1  // row groups per CTA (4: +8 ms of finalize under the ncu launch list, profiles/r02/s3c)
__global__ void __launch_bounds__(YF_R * 64) k_ytop_finalize(YtopParams p) {
    __shared__ double Ts[FT_NBMAX * FT_NBMAX];
    __shared__ double y0[YF_R][FT_NBMAX + 1];
    const int jb = threadIdx.x & 63, rl = threadIdx.x >> 6;
    const int ib = p.ib;
    const int halted = __ldcg(&p.ctl->halt);
    double tv[FT_NBMAX * FT_NBMAX / (YF_R * 64)];
#pragma unroll
    for (int u = 0; u < FT_NBMAX * FT_NBMAX / (YF_R * 64); u++) {
        const int i = threadIdx.x + u * YF_R * 64, a = i % FT_NBMAX, b = i / FT_NBMAX;
        tv[u] = (a < ib && b < ib) ? p.T[i] : 0.0;
    }
    if (halted) return;
#pragma unroll
    for (int u = 0; u < FT_NBMAX * FT_NBMAX / (YF_R * 64); u++) Ts[threadIdx.x + u * YF_R * 64] = tv[u];
    const int64_t st = (int64_t)(p.k + 1) * FT_NBMAX;
    double ey = 0.0;  // fused pre-update check: this thread's share of e^T Y(:, jb) over its rows
#pragma unroll 1
    for (int grp = 0; grp < YF_G; grp++) {
        const int row = (blockIdx.x * YF_G + grp) * YF_R + rl;
        if ((blockIdx.x * YF_G + grp) * YF_R > p.k) break;  // no row of this group exists (uniform)
        // this row's verify operands and the split partials: every load in flight together
        const bool vrow = p.verify && row <= p.k && jb == 0;
        const double a_k = vrow ? p.A[row + (int64_t)p.k * p.ldw] : 0.0;
        const double a_n = vrow ? p.A[row + (int64_t)p.n * p.ldw] : 0.0;
        const double f_r = vrow ? p.Fr[row] : 0.0;
        double acc = 0.0;
        if (row <= p.k && jb < ib) {
            // the split partials, 16 loads in flight at a time (fixed summation order)
            const double *src = p.ypart + (int64_t)row * FT_NBMAX + jb;
            for (int s0 = 0; s0 < p.nsplit; s0 += 16) {
                double v[16];
#pragma unroll
                for (int u = 0; u < 16; u++) v[u] = s0 + u < p.nsplit ? __ldcg(src + (int64_t)(s0 + u) * st) : 0.0;
#pragma unroll
                for (int u = 0; u < 16; u++) acc += v[u];
            }
        }
        __syncthreads();  // Ts written (first group) / the previous group's y0 reads are done
        y0[rl][jb] = acc;
        __syncthreads();
        double yv = 0.0;
        if (row <= p.k && jb < ib) {
            double y1 = 0.0, y2 = 0.0, y3 = 0.0;  // four independent chains
            int b = 0;
            for (; b + 3 <= jb; b += 4) {
                yv += y0[rl][b] * Ts[b + jb * FT_NBMAX];
                y1 += y0[rl][b + 1] * Ts[b + 1 + jb * FT_NBMAX];
                y2 += y0[rl][b + 2] * Ts[b + 2 + jb * FT_NBMAX];
                y3 += y0[rl][b + 3] * Ts[b + 3 + jb * FT_NBMAX];
            }
            for (; b <= jb; b++) yv += y0[rl][b] * Ts[b + jb * FT_NBMAX];
            yv = (yv + y1) + (y2 + y3);
            p.Y[row + (int64_t)jb * p.ldw] = yv;
            ey += yv;
        }
        if (vrow) {
            double rsum = 0.0;
            rsum = sum_strided(p.rowpart + row, p.k + 1, p.nsplit);
            rsum += a_k;
            if (p.ihi < p.n) rsum += sum_strided(p.A + row + (int64_t)p.ihi * p.ldw, p.ldw, p.n - p.ihi);
            double d = a_n - f_r - rsum;
            double tau_abs = p.ctl->c_thr * (double)p.n * 2.220446049250313e-16 * p.ctl->normF;
            if (not_within(d, tau_abs)) atomicAdd(&p.ctl->nflag, 1);
        }
    }
    if (!p.decide) return;
    // fused pre-update check (reading R15): e^T Y of rows 0..k, one add per column per CTA
    __syncthreads();
    y0[rl][jb] = ey;
    __syncthreads();
    if (rl == 0 && jb < ib) {
        double s = 0.0;
        for (int q = 0; q < YF_R; q++) s += y0[q][jb];
        atomicAdd(&p.ctl->eY[jb * FT_ESTR], s);
    }
    // the decision itself is taken by every CTA of the right update (GemmRightParams::pre_ctl)
}
int ft_ytop_rows_per_cta() { return YT_M; }
cudaError_t ft_launch_ytop(const YtopParams &p, cudaStream_t s) {
    static unsigned attr = 0;
    const unsigned dbit = ft_dev_bit();
    size_t smem = sizeof(YtopSmem);
    if (!(attr & dbit)) {
        cudaError_t e = cudaFuncSetAttribute(k_ytop_partial, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr |= dbit;
    }
    int nm = (p.k + 1 + YT_M - 1) / YT_M;
    g_ft_launches += 2;
    k_ytop_partial<<<dim3(nm, p.nsplit), YT_T, smem, s>>>(p);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    k_ytop_finalize<<<(p.k + 1 + YF_R * YF_G - 1) / (YF_R * YF_G), YF_R * 64, 0, s>>>(p);
    return cudaGetLastError();
}
