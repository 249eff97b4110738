// maxsub_kernels.cuh -- the O(1)-combine instance: maximum-subarray sum.
//
// T(n) = 2T(n/2) + O(1) with the segment summary
//   (tot, pre@pe, suf@ss, best@[bs,be])
// and the ordered, associative (NOT commutative) combine below (DESIGN.md
// Sec. 4, readings R9-R12).  Executed breadth-first like Alg 5
// except that neighbours are combined in order (left operand = lower
// indices): Alg 5's strided pairing a[id] + a[id+m] is only valid for a
// commutative combine.
//   NK4: every thread folds a contiguous chunk left to right (the leaves and
//        the bottom levels; exact by associativity), then ordered warp-shuffle
//        and cross-warp combines give one summary per CTA tile;
//   NK5: the last CTA to finish (atomic ticket) combines the tile summaries in
//        order: the top levels.
#pragma once
#include <cstdint>

#ifndef DC_MS_B4
#define DC_MS_B4 8
#endif

namespace dc {

// Identity ("empty segment") sentinel: |any real sum| <= 2^31 * 2^30 = 2^61.
constexpr long long kMsNeg = -(1LL << 62);

// Segment summary.  Inside a launch the indices are tile-local (int32);
// dc_maxsub_tuple (global, int64 indices) is used between CTAs and ranks.
template <class I>
struct MsTupT {
    long long tot, pre, suf, best;
    I pe, ss, bs, be;
};
using MsTup = MsTupT<int>;
using MsTupG = MsTupT<long long>;

template <class I>
__device__ __forceinline__ MsTupT<I> ms_empty() {
    MsTupT<I> t;
    t.tot = 0; t.pre = kMsNeg; t.suf = kMsNeg; t.best = kMsNeg;
    t.pe = 0; t.ss = 0; t.bs = 0; t.be = 0;
    return t;
}

// combine(L, R), L immediately left of R.
//   pre : keep L.pre on ties (smallest end)
//   suf : prefer R.tot + L.suf on ties (smallest start)
//   best: L.best, then the crossing (L.ss, R.pe), then R.best; a later
//         candidate replaces only if strictly larger (lexicographic order of
//         (start, end) follows candidate order).
template <class I>
__device__ __forceinline__ MsTupT<I> ms_combine(const MsTupT<I>& L, const MsTupT<I>& R) {
    MsTupT<I> c;
    c.tot = L.tot + R.tot;
    const long long lp = L.tot + R.pre;
    if (L.pre >= lp) { c.pre = L.pre; c.pe = L.pe; } else { c.pre = lp; c.pe = R.pe; }
    const long long rs = R.tot + L.suf;
    if (rs >= R.suf) { c.suf = rs; c.ss = L.ss; } else { c.suf = R.suf; c.ss = R.ss; }
    c.best = L.best; c.bs = L.bs; c.be = L.be;
    const long long cross = L.suf + R.pre;
    if (cross > c.best) { c.best = cross; c.bs = L.ss; c.be = R.pe; }
    if (R.best > c.best) { c.best = R.best; c.bs = R.bs; c.be = R.be; }
    return c;
}

// int32 -> FP64.  DC_MS_CVT = 1: 2^52 + 2^31 + x is the double with high word
// 0x43300000 and low word x ^ 0x80000000, so x = that - (2^52 + 2^31) exactly
// (one LOP3 + one DADD on the FP64 pipe instead of an I2F.F64 conversion).
#ifndef DC_MS_CVT
#define DC_MS_CVT 0
#endif
__device__ __forceinline__ double ms_i2d(int x) {
#if DC_MS_CVT
    return __hiloint2double(0x43300000, x ^ (int)0x80000000) - 4503601774854144.0;
#else
    return (double)x;
#endif
}

// Left-to-right fold of one element x at index i: combine(T, leaf(x, i)),
// which is Kadane's step with the tie rules above.  The running values are
// kept in FP64: a thread folds at most 2^16 int32 elements, so every real
// value is an integer of magnitude < 2^47 and FP64 adds and compares are
// EXACT (the sentinel -2^62 absorbs rounding and stays below every real value).  This moves the adds and compares onto the
// FP64 pipe and leaves only the selects on the integer ALU pipe, which the
// int64 version saturated.  tup() converts back to int64.
struct MsFold {
    double tot, pre, suf, best;
    int pe, ss, bs, be;
    __device__ __forceinline__ void init() {
        tot = 0.0; pre = (double)kMsNeg; suf = (double)kMsNeg; best = (double)kMsNeg;
        pe = ss = bs = be = 0;
    }
    __device__ __forceinline__ void step(int x, int i) {
        const double xd = ms_i2d(x);
        tot += xd;
        const bool up = tot > pre;                 // strict: smallest end
        pre = up ? tot : pre;
        pe = up ? i : pe;
        const bool restart = suf < 0.0;            // max(suf + x, x), ties keep suf
        suf = (restart ? 0.0 : suf) + xd;
        ss = restart ? i : ss;
        const bool better = suf > best;            // strict: smallest (start, end)
        best = better ? suf : best;
        bs = better ? ss : bs;
        be = better ? i : be;
    }
    // this = combine(this, R), R immediately right of this (ms_combine's rules
    // on the FP64 fields; exact for real values, the sentinel stays below all)
    __device__ __forceinline__ void absorb(const MsFold& R) {
        const double lp = tot + R.pre;
        const bool keep_pre = pre >= lp;
        const double rs = R.tot + suf;
        const bool left_suf = rs >= R.suf;
        const double cross = suf + R.pre;
        if (cross > best) { best = cross; bs = ss; be = R.pe; }
        if (R.best > best) { best = R.best; bs = R.bs; be = R.be; }
        pre = keep_pre ? pre : lp;
        pe = keep_pre ? pe : R.pe;
        suf = left_suf ? rs : R.suf;
        ss = left_suf ? ss : R.ss;
        tot += R.tot;
    }
    __device__ __forceinline__ MsTup tup() const {
        MsTup t;
        t.tot = (long long)tot; t.pre = (long long)pre; t.suf = (long long)suf;
        t.best = (long long)best;
        t.pe = pe; t.ss = ss; t.bs = bs; t.be = be;
        return t;
    }
};

template <class I>
__device__ __forceinline__ MsTupT<I> ms_shfl_down(const MsTupT<I>& t, int off) {
    MsTupT<I> r;
    r.tot = __shfl_down_sync(0xffffffffu, t.tot, off);
    r.pre = __shfl_down_sync(0xffffffffu, t.pre, off);
    r.suf = __shfl_down_sync(0xffffffffu, t.suf, off);
    r.best = __shfl_down_sync(0xffffffffu, t.best, off);
    r.pe = __shfl_down_sync(0xffffffffu, t.pe, off);
    r.ss = __shfl_down_sync(0xffffffffu, t.ss, off);
    r.bs = __shfl_down_sync(0xffffffffu, t.bs, off);
    r.be = __shfl_down_sync(0xffffffffu, t.be, off);
    return r;
}

// Ordered combine across the first `width` lanes (lane order == segment
// order); the result is valid in lane 0.
template <int WIDTH, class I>
__device__ __forceinline__ MsTupT<I> ms_warp_combine(MsTupT<I> t) {
#pragma unroll
    for (int off = 1; off < WIDTH; off <<= 1) {
        // branch-free (see ms_fold_warp): lanes that are not multiples of
        // 2*off compute unused values, and no shuffle is ever divergent
        const MsTupT<I> r = ms_shfl_down(t, off);
        t = ms_combine(t, r);
    }
    return t;
}

// Ordered combine of one tuple per thread of the CTA; result in thread 0.
template <int NT, class I>
__device__ __forceinline__ MsTupT<I> ms_block_combine(MsTupT<I> t, MsTupT<I>* red) {
    static_assert(NT / 32 <= 32, "one warp combines the warp results");
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    t = ms_warp_combine<32>(t);
    if (lane == 0) red[warp] = t;
    __syncthreads();
    if (warp == 0) {
        t = lane < NT / 32 ? red[lane] : ms_empty<I>();
        t = ms_warp_combine<NT / 32>(t);
    }
    return t;
}

__device__ __forceinline__ void ms_store(dc_maxsub_tuple* o, const MsTupG& t, long long off) {
    o->tot = t.tot; o->pre = t.pre; o->suf = t.suf; o->best = t.best;
    o->pe = t.pe + off; o->ss = t.ss + off; o->bs = t.bs + off; o->be = t.be + off;
}

__device__ __forceinline__ MsTupG ms_load(const dc_maxsub_tuple* o) {
    MsTupG t;
    t.tot = o->tot; t.pre = o->pre; t.suf = o->suf; t.best = o->best;
    t.pe = o->pe; t.ss = o->ss; t.bs = o->bs; t.be = o->be;
    return t;
}

// L2-coherent load of a summary written by another CTA of the same launch.
__device__ __forceinline__ MsTupG ms_load_cg(const dc_maxsub_tuple* o) {
    const long long* p = reinterpret_cast<const long long*>(o);
    MsTupG t;
    t.tot = __ldcg(p + 0); t.pre = __ldcg(p + 1); t.suf = __ldcg(p + 2); t.best = __ldcg(p + 3);
    t.pe = __ldcg(p + 4); t.ss = __ldcg(p + 5); t.bs = __ldcg(p + 6); t.be = __ldcg(p + 7);
    return t;
}

__device__ __forceinline__ MsTupG ms_widen(const MsTup& t, long long base) {
    MsTupG g;
    g.tot = t.tot; g.pre = t.pre; g.suf = t.suf; g.best = t.best;
    g.pe = t.pe + base; g.ss = t.ss + base; g.bs = t.bs + base; g.be = t.be + base;
    return g;
}

// NK4 + NK5.  Tiles of NT*C elements; CTA c folds the contiguous range of
// tiles [c*nt/G, (c+1)*nt/G) (G = gridDim.x, about one wave of resident
// CTAs), thread t folding the contiguous chunk [t*C, t*C+C) of each tile, and
// combines them in order into one summary.  The last CTA to finish (atomic
// ticket) combines the G summaries in order and writes either the result
// (mode 0) or the whole-array summary tuple (mode 1), indices offset by `off`.
template <int NT, int C>
__global__ void __launch_bounds__(NT)
nk4_maxsub(const int* __restrict__ x, long long n, dc_maxsub_tuple* __restrict__ parts,
           unsigned int* __restrict__ ticket, long long off, int mode,
           dc_maxsub_result* __restrict__ out_res, dc_maxsub_tuple* __restrict__ out_tup) {
    constexpr int TILE = NT * C;
    __shared__ MsTup red[NT / 32];
    __shared__ MsTupG redg[NT / 32];
    __shared__ bool am_last;
    const int tid = threadIdx.x;
    const long long ntiles = (n + TILE - 1) / TILE;
    const long long t0 = ntiles * blockIdx.x / gridDim.x;
    const long long t1 = ntiles * (blockIdx.x + 1) / gridDim.x;

    MsTupG acc = ms_empty<long long>();   // thread 0: this CTA's running summary
    for (long long tile = t0; tile < t1; ++tile) {
        const long long base = tile * TILE;
        const long long cbeg = base + (long long)tid * C;
        MsFold f;
        f.init();
        if (cbeg + C <= n) {
            // batches of 4*B4 elements (B4 x 128-bit loads in flight), the next
            // batch's loads issued before the current batch is folded
            constexpr int B4 = DC_MS_B4;
            static_assert(C % (4 * B4) == 0, "chunk must be whole batches");
            static_assert(C <= 256, "FP64 fold is exact only for chunks <= 2^8 elements");
            const int4* p4 = reinterpret_cast<const int4*>(x + cbeg);
            int4 v[B4], nv[B4];
#pragma unroll
            for (int q = 0; q < B4; ++q) v[q] = __ldg(p4 + q);
#pragma unroll 1
            for (int bt = 0; bt < C / (4 * B4); ++bt) {
                if (bt + 1 < C / (4 * B4)) {
#pragma unroll
                    for (int q = 0; q < B4; ++q) nv[q] = __ldg(p4 + (bt + 1) * B4 + q);
                }
                const int i0 = tid * C + bt * 4 * B4;   // tile-local index
#pragma unroll
                for (int q = 0; q < B4; ++q) {
                    f.step(v[q].x, i0 + 4 * q);
                    f.step(v[q].y, i0 + 4 * q + 1);
                    f.step(v[q].z, i0 + 4 * q + 2);
                    f.step(v[q].w, i0 + 4 * q + 3);
                }
#pragma unroll
                for (int q = 0; q < B4; ++q) v[q] = nv[q];
            }
        } else {
            for (long long e = cbeg; e < n && e < cbeg + C; ++e) f.step(x[e], (int)(e - base));
        }
        const MsTup t = ms_block_combine<NT>(f.tup(), red);
        if (tid == 0) acc = ms_combine(acc, ms_widen(t, base));
        __syncthreads();                           // red[] reused by the next tile
    }
    if (tid == 0) {
        ms_store(&parts[blockIdx.x], acc, 0);
        __threadfence();
        const unsigned int prev = atomicAdd(ticket, 1u);
        am_last = (prev == gridDim.x - 1);
    }
    __syncthreads();
    if (!am_last) return;

    // ---- NK5: ordered combine of the G part summaries (top levels)
    __threadfence();
    const int np = gridDim.x;
    const int per = (np + NT - 1) / NT;
    MsTupG a = ms_empty<long long>();
    for (int q = tid * per; q < min(np, tid * per + per); ++q) a = ms_combine(a, ms_load_cg(parts + q));
    a = ms_block_combine<NT>(a, redg);
    if (tid == 0) {
        if (mode == 0) {
            out_res->sum = a.best;
            out_res->start = a.bs + off;
            out_res->end = a.be + off;
        } else {
            ms_store(out_tup, a, off);
        }
        *ticket = 0u;   // re-arm for the next launch on this plan
    }
}

// Ordered combine of `count` summaries (multi-GPU: one per rank, rank order).
__global__ void nk5_combine_tuples(const dc_maxsub_tuple* __restrict__ tups, int count,
                                   dc_maxsub_result* __restrict__ out) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    MsTupG acc = ms_empty<long long>();
    for (int q = 0; q < count; ++q) acc = ms_combine(acc, ms_load(tups + q));
    out->sum = acc.best;
    out->start = acc.bs;
    out->end = acc.be;
}

}  // namespace dc
