// maxsub_rows.cuh -- NK4 with every lane folding ONE contiguous row (-DDC_MS_ROWS=1;
// measured no faster than the warp-segment kernel).
//
// Same method as nk4_maxsub / nk4_maxsub_tma: contiguous pieces are folded
// left to right (the leaves and the bottom levels of the D&C tree, exact by
// associativity of the O(1) combine), then combined in order (the top levels:
// lane -> warp -> CTA -> last CTA).  What changes is the data layout.  The
// array is viewed as a 2-D tensor of rows of W elements (W = ceil(n / lanes),
// rounded up to 16 bytes; row r = elements [r*W, (r+1)*W)), and lane l of
// warp w owns row 32*w + l: it folds its whole row as ONE running summary.
// Rows arrive by 2-D TMA tensor copies (cp.async.bulk.tensor.2d): one copy
// brings a box of L columns x 32 rows -- the next L elements of every lane's
// row -- into an S-stage shared-memory ring (mbarrier per warp and stage), so
// one instruction feeds the whole warp and no lane's data is interleaved with
// another's.  Compared with the warp-segment layout of nk4_maxsub_tma (each
// segment = 32 lanes x L consecutive elements), the per-segment ordered warp
// tree (5 shuffle levels of an 8-field tuple, ~230 instructions per segment)
// disappears: the warp tree runs once per warp.  Without that per-segment
// cost the segments can be short, so the ring is small and three CTAs fit on
// an SM (24 warps instead of 8 to hide the fold's dependency latency).
//
// The elements after the last full row (fewer than W) are folded by warp 0 of
// the last CTA and appended in order.  Exactness: a lane folds at most W <=
// 2^16 int32 values, so every FP64 running value is an integer below 2^47
// (MsFold, maxsub_kernels.cuh).
#pragma once
#include <cuda.h>

#include <cstdint>

#include "maxsub_kernels.cuh"
#include "sort_kernels.cuh"

namespace dc {

__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* map, int c0, int c1,
                                            uint32_t bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(bar)
        : "memory");
}

// Ordered warp fold of a per-lane MsFold (lane order = row order); lane 0.
__device__ __forceinline__ MsFold ms_fold_rows_warp(MsFold t) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        MsFold r;
        r.tot = __shfl_down_sync(0xffffffffu, t.tot, off);
        r.pre = __shfl_down_sync(0xffffffffu, t.pre, off);
        r.suf = __shfl_down_sync(0xffffffffu, t.suf, off);
        r.best = __shfl_down_sync(0xffffffffu, t.best, off);
        r.pe = __shfl_down_sync(0xffffffffu, t.pe, off);
        r.ss = __shfl_down_sync(0xffffffffu, t.ss, off);
        r.bs = __shfl_down_sync(0xffffffffu, t.bs, off);
        r.be = __shfl_down_sync(0xffffffffu, t.be, off);
        if ((lane & (2 * off - 1)) == 0) t.absorb(r);
    }
    return t;
}

// Geometry of a launch: rows of W elements, nrows full rows, the tail
// [nrows * W, n) folded separately.
struct MsRows {
    long long n, W, nrows;
};

template <int NT, int L, int S, int MINB>
__global__ void __launch_bounds__(NT, MINB)
nk4_maxsub_rows(const __grid_constant__ CUtensorMap tmap, const int* __restrict__ x, MsRows g,
                dc_maxsub_tuple* __restrict__ parts, unsigned int* __restrict__ ticket,
                long long off, int mode, dc_maxsub_result* __restrict__ out_res,
                dc_maxsub_tuple* __restrict__ out_tup) {
    static_assert(L % 4 == 0 && ((L / 4) & 1) == 1, "row stride in the ring: 4 x odd words");
    constexpr int NW = NT / 32;
    constexpr int BOX = 32 * L;                                // elements per warp and stage
    constexpr int V = L / 4;
    extern __shared__ __align__(128) int ms_ring[];           // [S][NW][32][L]
    __shared__ __align__(8) uint64_t bars[S][NW];
    __shared__ MsTup red[NW];
    __shared__ MsTupG redg[NW];
    __shared__ bool am_last;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

    const long long row0 = ((long long)blockIdx.x * NW + warp) * 32;   // this warp's first row
    const long long crow = (long long)blockIdx.x * NW * 32;              // this CTA's first row
    const long long cbase = min(g.n, crow * g.W);                        // CTA-local index base
    const bool warp_live = row0 < g.nrows;
    const long long myrow = row0 + lane;
    const bool live = myrow < g.nrows;
    const int nseg = warp_live ? (int)((g.W + L - 1) / L) : 0;

    if (lane == 0) {
#pragma unroll
        for (int s = 0; s < S; ++s) mbar_init(smem_addr(&bars[s][warp]), 1);
    }
    __syncwarp();
    auto stage = [&](int s) { return ms_ring + (s * NW + warp) * BOX; };
    auto issue = [&](int k) {          // lane 0: columns [k*L, k*L + L) of the warp's 32 rows
        const int s = k % S;
        const uint32_t bar = smem_addr(&bars[s][warp]);
        mbar_arrive_expect_tx(bar, 4u * BOX);                  // the whole box (OOB: zeros)
        tma_load_2d(smem_addr(stage(s)), &tmap, k * L, (int)row0, bar);
    };
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < S; ++k)
            if (k < nseg) issue(k);
    }

    MsFold acc;
    acc.init();
    const int ibase = (int)(myrow * g.W - cbase);              // CTA-local index of my row
    for (int k = 0; k < nseg; ++k) {
        const int s = k % S;
        mbar_wait(smem_addr(&bars[s][warp]), (uint32_t)((k / S) & 1));
        const int* sl = stage(s) + lane * L;
        const long long c0 = (long long)k * L;
        const int cnt = (int)min((long long)L, g.W - c0);
        const int i0 = ibase + (int)c0;
        if (live) {
            if (cnt == L) {
#pragma unroll
                for (int q = 0; q < V; ++q) {
                    const int4 v = *reinterpret_cast<const int4*>(sl + 4 * q);
                    acc.step(v.x, i0 + 4 * q);
                    acc.step(v.y, i0 + 4 * q + 1);
                    acc.step(v.z, i0 + 4 * q + 2);
                    acc.step(v.w, i0 + 4 * q + 3);
                }
            } else {
                for (int e = 0; e < cnt; ++e) acc.step(sl[e], i0 + e);
            }
        }
        __syncwarp();                                          // every lane is done with stage s
        if (lane == 0 && k + S < nseg) {
            fence_proxy_async_smem();
            issue(k + S);
        }
    }
    acc = ms_fold_rows_warp(acc);

    // ---- warps -> CTA summary (thread 0), in order
    if (lane == 0) red[warp] = acc.tup();
    __syncthreads();
    if (tid == 0) {
        MsTupG c = ms_empty<long long>();
        for (int w = 0; w < NW; ++w) c = ms_combine(c, ms_widen(red[w], cbase));
        ms_store(&parts[blockIdx.x], c, 0);
        __threadfence();
        am_last = atomicAdd(ticket, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!am_last) return;

    // ---- NK5: ordered combine of the per-CTA summaries (top levels), then the tail
    __threadfence();
    const int np = gridDim.x;
    const int per = (np + NT - 1) / NT;
    MsTupG a = ms_empty<long long>();
    for (int q = tid * per; q < min(np, tid * per + per); ++q) a = ms_combine(a, ms_load_cg(parts + q));
    a = ms_block_combine<NT>(a, redg);
    const long long t0 = g.nrows * g.W;                        // tail [t0, n): < W elements
    if (t0 < g.n) {
        __shared__ MsTupG s_tail;
        if (warp == 0) {
            const long long len = g.n - t0;
            const long long per_l = (len + 31) / 32;
            const long long b = t0 + lane * per_l, e = min(g.n, b + per_l);
            MsFold f;
            f.init();
            for (long long j = b; j < e; ++j) f.step(x[j], (int)(j - t0));
            f = ms_fold_rows_warp(f);
            if (lane == 0) s_tail = ms_widen(f.tup(), t0);
        }
        __syncthreads();
        if (tid == 0) a = ms_combine(a, s_tail);
    }
    if (tid == 0) {
        if (mode == 0) {
            out_res->sum = a.best;
            out_res->start = a.bs + off;
            out_res->end = a.be + off;
        } else {
            ms_store(out_tup, a, off);
        }
        *ticket = 0u;
    }
}

}  // namespace dc
