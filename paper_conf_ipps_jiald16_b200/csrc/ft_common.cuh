// ft_common.cuh -- device helpers shared by the ftgehrd kernels (product path).
// No code here is shared with oracle/ (the CPU oracle is a separate program).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#ifndef FT_NBMAX
#define FT_NBMAX 64  // max panel width (opts.nb <= 64)
#endif
#ifndef FT_DPMAX
#define FT_DPMAX 160  // deterministic mode: max CTAs per panel launch (rank group)
#endif
#define FT_KPAD (FT_NBMAX + 4)  // smem row stride for K <= 64 operands (conflict-free DMMA frags)

#define FT_DEV __device__ __forceinline__

// ---------------------------------------------------------------------------
// FP64 tensor-core MMA (sm_80+ mma.sync f64; lowers to DMMA on sm_100a).
// D(8x8) += A(8x4, row) * B(4x8, col).  Fragment ownership (lane l):
//   A: a = A[l/4][l%4]      B: b = B[l%4][l/4]      C/D: d0,d1 = C[l/4][2(l%4)+{0,1}]
// ---------------------------------------------------------------------------
FT_DEV void dmma_8x8x4(double &d0, double &d1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(d0), "+d"(d1)
                 : "d"(a), "d"(b));
}

// Warp-level tile MMA: acc[MI][NI] (8MI x 8NI) += A(8MI x K) * B(K x 8NI).
// A element (m,k) at As[m*SA + k] (AK = false) or As[k*SA + m] (AK = true).
// B element (k,n) at Bs[n*SB + k].  K is a multiple of 4; m0/n0 are the warp
// tile origin inside the smem tiles.
template <int MI, int NI, bool AK>
FT_DEV void warp_mma(double (&acc)[MI][NI][2], const double *As, int SA, const double *Bs, int SB,
                     int m0, int n0, int K) {
    const int lane = threadIdx.x & 31;
    const int lr = lane >> 2, lc = lane & 3;
#pragma unroll 2
    for (int k = 0; k < K; k += 4) {
        double a[MI], b[NI];
#pragma unroll
        for (int mi = 0; mi < MI; mi++) {
            int m = m0 + mi * 8 + lr;
            a[mi] = AK ? As[(k + lc) * SA + m] : As[m * SA + k + lc];
        }
#pragma unroll
        for (int ni = 0; ni < NI; ni++) {
            int nn = n0 + ni * 8 + lr;
            b[ni] = Bs[nn * SB + k + lc];
        }
#pragma unroll
        for (int mi = 0; mi < MI; mi++)
#pragma unroll
            for (int ni = 0; ni < NI; ni++) dmma_8x8x4(acc[mi][ni][0], acc[mi][ni][1], a[mi], b[ni]);
    }
}

// Same with both operand layouts selectable: A(m,k) at As[m*SA+k] (AK=false) or
// As[k*SA+m] (AK=true); B(k,n) at Bs[n*SB+k] (BK=false) or Bs[k*SB+n] (BK=true).
// With strides = 4 (mod 16) doubles every fragment load is bank-conflict free.
template <int MI, int NI, bool AK, bool BK>
FT_DEV void warp_mma2(double (&acc)[MI][NI][2], const double *As, int SA, const double *Bs, int SB, int m0,
                      int n0, int K) {
    const int lane = threadIdx.x & 31;
    const int lr = lane >> 2, lc = lane & 3;
#pragma unroll 4
    for (int k = 0; k < K; k += 4) {
        double a[MI], b[NI];
#pragma unroll
        for (int mi = 0; mi < MI; mi++) {
            int m = m0 + mi * 8 + lr;
            a[mi] = AK ? As[(k + lc) * SA + m] : As[m * SA + k + lc];
        }
#pragma unroll
        for (int ni = 0; ni < NI; ni++) {
            int nn = n0 + ni * 8 + lr;
            b[ni] = BK ? Bs[(k + lc) * SB + nn] : Bs[nn * SB + k + lc];
        }
#pragma unroll
        for (int mi = 0; mi < MI; mi++)
#pragma unroll
            for (int ni = 0; ni < NI; ni++) dmma_8x8x4(acc[mi][ni][0], acc[mi][ni][1], a[mi], b[ni]);
    }
}

// 16-byte asynchronous global->shared copy (LDGSTS); src_bytes < 16 zero-fills the tail
FT_DEV void cp_async16(void *smem, const void *gmem, int src_bytes) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem), "r"(src_bytes) : "memory");
}
// 8-byte asynchronous global->shared copy (LDGSTS); src_bytes = 0 zero-fills
FT_DEV void cp_async8(void *smem, const void *gmem, int src_bytes) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(s), "l"(gmem), "r"(src_bytes) : "memory");
}
FT_DEV void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
FT_DEV void cp_async_wait() {
    asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory");
}

// ---------------------------------------------------------------------------
// Bulk asynchronous copies (the TMA unit's 1-D cp.async.bulk, SASS UBLKCP) completing on an
// mbarrier transaction count: one lane moves a whole contiguous column segment of an operand tile
// into its (padded, bank-conflict-free) row of shared memory.  src, dst 16-byte aligned, bytes a
// multiple of 16.
// ---------------------------------------------------------------------------
FT_DEV unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
FT_DEV void mbar_init(unsigned long long *bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
FT_DEV void mbar_fence_init() { asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory"); }
// generic-proxy accesses of this thread (made visible by a preceding bar.sync) before async-proxy writes
FT_DEV void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory"); }
FT_DEV void mbar_expect_tx(unsigned long long *bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
FT_DEV void bulk_g2s(void *dst, const void *src, unsigned bytes, unsigned long long *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
// consumer release of a pipeline buffer (the arrive orders this thread's earlier shared-memory
// reads before the producer's next async-proxy write into the buffer, as in a TMA pipeline)
FT_DEV void mbar_arrive(unsigned long long *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
// 2-D tensor TMA (SASS UTMALDG): the box at element coordinates (c0 = row, c1 = column) of the
// tensor map `map` (a __grid_constant__ kernel parameter) into shared memory at dst (128-byte
// aligned), completing on bar's transaction count; out-of-bounds elements are zero-filled
FT_DEV void tma_load_2d(void *dst, const void *map, int c0, int c1, unsigned long long *bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], "
        "[%4];\n" ::"r"(smem_u32(dst)),
        "l"(map), "r"(c0), "r"(c1), "r"(smem_u32(bar))
        : "memory");
}
FT_DEV void tma_prefetch_map(const void *map) {
    asm volatile("prefetch.tensormap [%0];\n" ::"l"(map) : "memory");
}
FT_DEV void mbar_wait(unsigned long long *bar, unsigned parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

// element coordinates owned by this lane in fragment (mi, ni), v = 0/1
FT_DEV int frag_row(int mi) { return mi * 8 + ((threadIdx.x & 31) >> 2); }
FT_DEV int frag_col(int ni, int v) { return ni * 8 + 2 * (threadIdx.x & 3) + v; }

// ---------------------------------------------------------------------------
// Grid barrier for a cooperative (co-resident) launch: monotonic arrival
// counter, release/acquire at gpu scope.  `epoch` counts barriers passed by
// this CTA; the counter must be zero at launch.
// ---------------------------------------------------------------------------
FT_DEV unsigned ld_acquire_u32(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];\n" : "=r"(v) : "l"(p) : "memory");
    return v;
}
FT_DEV void red_release_add_u32(unsigned *p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;\n" ::"l"(p), "r"(v) : "memory");
}
// last-CTA-done counters: one acq_rel atomic replaces fence + atomic + fence (the release is
// cumulative over the CTA's writes ordered before it by bar.sync, the acquire over the last
// CTA's reads ordered after it by the next bar.sync)
FT_DEV int atom_add_acqrel_s32(int *p, int v) {
    int old;
    asm volatile("atom.acq_rel.gpu.global.add.s32 %0, [%1], %2;\n" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}
FT_DEV void grid_barrier(unsigned *count, unsigned &epoch, unsigned nblocks) {
    __syncthreads();
    if (threadIdx.x == 0) {
        epoch += 1;
        const unsigned target = epoch * nblocks;
        // release is cumulative over the CTA's writes ordered before it by bar.sync;
        // the acquire load orders everything after it (PTX memory model)
        red_release_add_u32(count, 1u);
        while (ld_acquire_u32(count) < target) {
        }
    }
    __syncthreads();
}

// Watchdog for spins on flags written by OTHER GPUs (multi-rank exchanges): a peer that never
// arrives (a dead rank, a broken peer mapping) ends the kernel with a trap after 60 s -- the call
// then fails with a CUDA error instead of hanging the job.  Cheap: the timer is read once per 1024
// polls.
FT_DEV void peer_spin_guard(unsigned long long &t0, unsigned &polls) {
    if ((++polls & 1023u) != 0u) return;
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t0 == 0ull) t0 = t;
    else if (t - t0 > 60ull * 1000000000ull) __trap();
}

// L2-coherent loads for data written by other CTAs inside the same launch
FT_DEV double ldcg(const double *p) { return __ldcg(p); }

// sum_{i < N} p[i * stride] (L2-coherent loads), eight loads in flight at a time; fixed
// summation order for a given N (deterministic)
FT_DEV double sum_strided(const double *p, int64_t stride, int N) {
    double s0 = 0.0, s1 = 0.0, s2 = 0.0, s3 = 0.0;
    int i = 0;
    for (; i + 8 <= N; i += 8) {
        double v[8];
#pragma unroll
        for (int u = 0; u < 8; u++) v[u] = __ldcg(p + (int64_t)(i + u) * stride);
        s0 += v[0] + v[4];
        s1 += v[1] + v[5];
        s2 += v[2] + v[6];
        s3 += v[3] + v[7];
    }
    if (i < N) {  // remainder: one predicated batch (all loads in flight together)
        double v[8];
#pragma unroll
        for (int u = 0; u < 8; u++) v[u] = i + u < N ? __ldcg(p + (int64_t)(i + u) * stride) : 0.0;
        s0 += v[0] + v[4];
        s1 += v[1] + v[5];
        s2 += v[2] + v[6];
        s3 += v[3] + v[7];
    }
    return (s0 + s1) + (s2 + s3);
}

// Deterministic sums of CTA partials (opts.deterministic): out[v] = the sum over the P CTAs of
// accumulator idx(v) of one set, idx running over [a0, a0+n0) then [a1, a1+n1) then [a2, a2+n2);
// part points at the set's block of [FT_ACC_STRIDE][FT_DPMAX] partials.  Warp w takes values
// w, w + nw, ... four at a time (all their loads in flight), lane l the CTAs l, l + 32, ... in
// order, then a fixed xor tree: the same additions in the same order on every call and in every
// CTA.  Called by every thread of the CTA; a __syncthreads must follow before out is read.
FT_DEV void det_sum(const double *part, int P, int a0, int n0, int a1, int n1, int a2, int n2, double *out) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const int nv = n0 + n1 + n2;
    for (int v0 = w; v0 < nv; v0 += 4 * nw) {
        double s[4];
#pragma unroll
        for (int u = 0; u < 4; u++) {
            const int v = v0 + u * nw;
            s[u] = 0.0;
            if (v < nv) {
                const int idx = v < n0 ? a0 + v : (v < n0 + n1 ? a1 + (v - n0) : a2 + (v - n0 - n1));
                const double *q = part + (int64_t)idx * FT_DPMAX;
                double x[(FT_DPMAX + 31) / 32];
#pragma unroll
                for (int b = 0; b < (FT_DPMAX + 31) / 32; b++) x[b] = lane + 32 * b < P ? __ldcg(q + lane + 32 * b) : 0.0;
#pragma unroll
                for (int b = 0; b < (FT_DPMAX + 31) / 32; b++) s[u] += x[b];
            }
        }
#pragma unroll
        for (int u = 0; u < 4; u++) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) s[u] += __shfl_xor_sync(0xffffffffu, s[u], o);
            const int v = v0 + u * nw;
            if (lane == 0 && v < nv) out[v] = s[u];
        }
    }
}

FT_DEV double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

FT_DEV bool not_within(double d, double tau) { return !(fabs(d) <= tau); }  // NaN -> true

// Checksum of row r of the block-reflector factor T over the entries the updates read (the upper
// triangle, T(r, c) for r <= c < K; reading R15 extended to T).  Four consecutive lanes
// per row (q = 0..3 takes c = r+q, r+q+4, ...), combined by xor shuffles: the same additions in
// the same order wherever it is evaluated, so a fault-free recomputation matches the checksum the
// panel stored.  get(r, c) returns T(r, c); every lane of the 4-lane group must call it.
template <class F>
FT_DEV void t_row_checksum(F get, int r, int q, int K, double &s, double &sa) {
    s = 0.0;
    sa = 0.0;
    if (r < K)
        for (int c = r + q; c < K; c += 4) {
            const double v = get(r, c);
            s += v;
            sa += fabs(v);
        }
    s += __shfl_xor_sync(0xffffffffu, s, 1);
    sa += __shfl_xor_sync(0xffffffffu, sa, 1);
    s += __shfl_xor_sync(0xffffffffu, s, 2);
    sa += __shfl_xor_sync(0xffffffffu, sa, 2);
}
