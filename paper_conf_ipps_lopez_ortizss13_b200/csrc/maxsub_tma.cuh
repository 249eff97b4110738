// maxsub_tma.cuh -- NK4 with TMA-streamed warp segments (the default NK4).
//
// Same method as nk4_maxsub (maxsub_kernels.cuh): contiguous pieces are
// folded left to right (leaves + bottom levels), then combined in order
// (top levels).  What changes is how the data arrives.  Loading a private
// contiguous chunk per lane with 128-bit loads makes every warp load touch
// 32 lines (32 L1 requests per instruction; the L1/TEX pipe bounded that
// kernel), and one TMA copy per lane costs a request per 256 bytes.  Here
// every WARP owns one contiguous range and streams it in segments of 32*L
// elements, one 1-D TMA bulk copy per segment (S-stage ring, one mbarrier per
// warp and stage); lane l folds the L contiguous elements [l*L, (l+1)*L) of
// the segment from shared memory (L/4 odd: the 128-bit reads of a warp are
// bank-conflict free) as J interleaved chains, and an ordered FP64 warp tree
// folds the 32 lane summaries into the warp's running summary.  Warps, then
// CTAs (atomic ticket, last CTA), are combined in order as before.
//
// VO (values-only, the default since r02b; -DDC_MS_VONLY=0 keeps the indexed
// fold): the per-element fold keeps only the four
// values (tot, pre, suf, best: two DADDs and three max) and no indices; each
// lane's L-element chunk then enters the ordered combine as one leaf labelled
// by its chunk start.  The combine's tie rules pick the lexicographically
// smallest (start chunk, end chunk) pair, and that pair holds the
// lexicographically smallest optimal (start, end) (reading R21), so
// the last CTA recovers the exact element indices by re-scanning at most
// four chunks (ms_recover).
#pragma once
#include <cstdint>

#include "maxsub_kernels.cuh"
#include "sort_kernels.cuh"

namespace dc {

// Timeline probe (tools/nk4_trace.cu only): %globaltimer at CTA entry, after
// each warp's segment loop, after the CTA's ticket, and at the end of the last
// CTA, into the __device__ array dc::dc_ms_trace the tool defines before
// including this header.
#ifdef DC_MS_TRACE
#define DC_MS_TRACE_AT(slot)                                                      \
    do {                                                                          \
        unsigned long long t_;                                                    \
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                    \
        dc_ms_trace[slot] = t_;                                                   \
    } while (0)
#else
#define DC_MS_TRACE_AT(slot) do { } while (0)
#endif

__device__ __forceinline__ MsFold ms_fold_shfl_down(const MsFold& t, int off) {
    MsFold r;
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

// Ordered combine of the 32 lanes' folds (lane order = segment order); lane 0.
// Branch-free: every lane absorbs its partner at every level.  Only lanes
// with (lane & (2*off - 1)) == 0 hold a meaningful summary afterwards (the
// partner they read at the next level is again such a lane), the others carry
// unused values.  A conditional absorb made the next level's full-mask
// shuffles potentially divergent, and the compiler guarded every level with a
// WARPSYNC / BRA.DIV fallback path (~45 extra instructions per level, ~30 %
// of NK4's instructions were the per-segment tree).
__device__ __forceinline__ MsFold ms_fold_warp(MsFold t) {
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const MsFold r = ms_fold_shfl_down(t, off);
        t.absorb(r);
    }
    return t;
}

// Values-only fold of one chunk (no indices).  Same FP64 exactness argument
// as MsFold; the maxima reproduce the strict/tie rules' values (only the
// indices depend on ties, and those are recovered separately).  Maxima are
// compare-and-select (DSETP + FSEL pairs): fmax's NaN semantics lower to
// DSETP.MAX + SEL + FSEL + a predicated LOP3 plus register moves (measured
// 48 vs 29 us per launch in r01), and the operands here are never NaN.
__device__ __forceinline__ double dmax(double a, double b) {
    double r;
    asm("{\n\t.reg .pred p;\n\tsetp.gt.f64 p, %1, %2;\n\tselp.f64 %0, %1, %2, p;\n\t}"
        : "=d"(r) : "d"(a), "d"(b));
    return r;
}
struct MsVal {
    double tot, pre, suf, best;
    __device__ __forceinline__ void init() {
        tot = 0.0; pre = (double)kMsNeg; suf = (double)kMsNeg; best = (double)kMsNeg;
    }
    __device__ __forceinline__ void step(int x) {
        const double xd = ms_i2d(x);
        tot += xd;
        pre = dmax(pre, tot);
        suf = dmax(suf, 0.0) + xd;
        best = dmax(best, suf);
    }
    __device__ __forceinline__ void absorb(const MsVal& R) {   // R right of this
        best = dmax(best, dmax(suf + R.pre, R.best));
        pre = dmax(pre, tot + R.pre);
        suf = dmax(R.tot + suf, R.suf);
        tot += R.tot;
    }
};

// Warp-parallel scans over one staged chunk s[0, len) (len <= L): lane l owns
// the E = ceil(L/32) elements [l*E, l*E + E).  Prefix sums P_j = s[0] + ...
// + s[j] in int64 (exact); an exclusive warp scan of the lane totals gives
// every lane its offset.
template <int L>
struct MsChunkScan {
    static constexpr int E = (L + 31) / 32;
    long long p[E];   // P_j of this lane's elements (j < len)
    int len;
    __device__ __forceinline__ MsChunkScan(const int* s, int len_) : len(len_) {
        const int lane = threadIdx.x & 31;
        long long run = 0;
#pragma unroll
        for (int t = 0; t < E; ++t) {
            const int j = lane * E + t;
            run += j < len ? s[j] : 0;
            p[t] = run;
        }
        long long inc = run;                       // inclusive scan of lane totals
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const long long u = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += u;
        }
        const long long off = inc - run;
#pragma unroll
        for (int t = 0; t < E; ++t) p[t] += off;
    }
};
// (value, index) reductions over the warp; ties -> smallest index.
__device__ __forceinline__ void ms_warp_argmax(long long& v, int& i) {
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        const long long ov = __shfl_xor_sync(0xffffffffu, v, o);
        const int oi = __shfl_xor_sync(0xffffffffu, i, o);
        if (ov > v || (ov == v && oi < i)) { v = ov; i = oi; }
    }
}
__device__ __forceinline__ void ms_warp_argmin(long long& v, int& i) {
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        const long long ov = __shfl_xor_sync(0xffffffffu, v, o);
        const int oi = __shfl_xor_sync(0xffffffffu, i, o);
        if (ov < v || (ov == v && oi < i)) { v = ov; i = oi; }
    }
}
// smallest e maximising P_e (the prefix end)
template <int L>
__device__ int ms_par_first_max_prefix(const MsChunkScan<L>& c) {
    const int lane = threadIdx.x & 31;
    long long v = kMsNeg;
    int i = 1 << 30;
#pragma unroll
    for (int t = 0; t < MsChunkScan<L>::E; ++t) {
        const int j = lane * MsChunkScan<L>::E + t;
        if (j < c.len && c.p[t] > v) { v = c.p[t]; i = j; }
    }
    ms_warp_argmax(v, i);
    return i;
}
// smallest start k maximising the suffix sum = smallest k minimising P_{k-1}
// over k - 1 in [-1, len - 2] (P_{-1} = 0)
template <int L>
__device__ int ms_par_first_max_suffix(const MsChunkScan<L>& c) {
    const int lane = threadIdx.x & 31;
    long long v = 0;                          // P_{-1} = 0 at k = 0 (lane 0 only)
    int i = lane == 0 ? 0 : (1 << 30);
    if (lane != 0) v = -kMsNeg;
#pragma unroll
    for (int t = 0; t < MsChunkScan<L>::E; ++t) {
        const int j = lane * MsChunkScan<L>::E + t;
        if (j + 1 < c.len && (c.p[t] < v || (c.p[t] == v && j + 1 < i))) { v = c.p[t]; i = j + 1; }
    }
    ms_warp_argmin(v, i);
    return i;
}
// lexicographically smallest (s, e) maximising sum(s..e) inside the chunk:
// s_e = first argmin of Q_q = P_{q-1} over q in [0, e], e = first argmax of
// P_e - Q_{s_e} (R21: that pair is the lexicographic minimum)
template <int L>
__device__ void ms_par_kadane(const MsChunkScan<L>& c, const int* s, int& bs, int& be) {
    constexpr int E = MsChunkScan<L>::E;
    const int lane = threadIdx.x & 31;
    long long q[E];
    int qi[E];
    long long mn = -kMsNeg;                   // lane-local inclusive prefix min of Q
    int mi = 1 << 30;
#pragma unroll
    for (int t = 0; t < E; ++t) {
        const int j = lane * E + t;
        const long long Q = j < c.len ? c.p[t] - s[j] : -kMsNeg;   // P_{j-1}
        if (Q < mn) { mn = Q; mi = j; }
        q[t] = mn;
        qi[t] = mi;
    }
    // exclusive warp scan of the lane minima (ties keep the earlier index)
    long long em = mn;
    int ei = mi;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const long long um = __shfl_up_sync(0xffffffffu, em, o);
        const int ui = __shfl_up_sync(0xffffffffu, ei, o);
        if (lane >= o && (um < em || (um == em && ui < ei))) { em = um; ei = ui; }
    }
    long long pm = __shfl_up_sync(0xffffffffu, em, 1);
    int pi = __shfl_up_sync(0xffffffffu, ei, 1);
    if (lane == 0) { pm = -kMsNeg; pi = 1 << 30; }
    long long v = kMsNeg;
    int e = 1 << 30, sb = 0;
#pragma unroll
    for (int t = 0; t < E; ++t) {
        const int j = lane * E + t;
        long long m = q[t];
        int mi2 = qi[t];
        if (pm < m || (pm == m && pi < mi2)) { m = pm; mi2 = pi; }   // earlier lanes first
        if (j < c.len) {
            const long long val = c.p[t] - m;
            if (val > v) { v = val; e = j; sb = mi2; }
        }
    }
    int ee = e;
    ms_warp_argmax(v, ee);                     // first e with the maximum value
    bs = __shfl_sync(0xffffffffu, sb, ee / E);
    be = ee;
}

// Exact indices from chunk labels (warp 0 of the last CTA).  a's pe/ss/bs/be
// are chunk starts; on return they are element indices.  pe: first prefix
// maximum inside its chunk; ss: first suffix maximum inside its chunk; best:
// the in-chunk maximum subarray when start and end chunk coincide, else the
// suffix-start / prefix-end scans of the two.  The (at most four) chunks are
// staged in shared memory by coalesced warp loads; every scan is a warp-
// parallel int64 prefix scan with (value, index) reductions (r01's serial
// scans of global memory cost ~17 us, r02's serial scans of shared memory
// ~2-3 us on the critical path).
template <int L>
__device__ void ms_recover(const int* __restrict__ x, long long n, MsTupG& a, long long* rec) {
    __shared__ int stage[4][L];
    const int lane = threadIdx.x & 31;
    const long long cs[4] = {a.pe, a.ss, a.bs, a.be};
#pragma unroll
    for (int q = 0; q < 4; ++q)
        for (int e = lane; e < L; e += 32)
            if (cs[q] + e < n) stage[q][e] = x[cs[q] + e];
    __syncwarp();
    int len[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) len[q] = (int)min((long long)L, n - cs[q]);
    const MsChunkScan<L> c0(stage[0], len[0]);
    const long long pe = a.pe + ms_par_first_max_prefix<L>(c0);
    const MsChunkScan<L> c1(stage[1], len[1]);
    const long long ss = a.ss + ms_par_first_max_suffix<L>(c1);
    const MsChunkScan<L> c2(stage[2], len[2]);
    long long bs, be;
    if (a.bs == a.be) {
        int s0, e0;
        ms_par_kadane<L>(c2, stage[2], s0, e0);
        bs = a.bs + s0;
        be = a.bs + e0;
    } else {
        bs = a.bs + ms_par_first_max_suffix<L>(c2);
        const MsChunkScan<L> c3(stage[3], len[3]);
        be = a.be + ms_par_first_max_prefix<L>(c3);
    }
    (void)rec;
    a.pe = pe; a.ss = ss; a.bs = bs; a.be = be;
}

template <int NT, int L, int S, int J, bool VO>
__global__ void __launch_bounds__(NT, 1)
nk4_maxsub_tma(const int* __restrict__ x, long long n, long long RW,
               dc_maxsub_tuple* __restrict__ parts, unsigned int* __restrict__ ticket,
               long long off, int mode, dc_maxsub_result* __restrict__ out_res,
               dc_maxsub_tuple* __restrict__ out_tup) {
    static_assert(L % 4 == 0 && ((L / 4) & 1) == 1, "lane stride: 4 x odd words");
    constexpr int NW = NT / 32;
    constexpr int SEG = 32 * L;                                // elements per segment
    constexpr int V = L / 4;                                   // 16-byte vectors per lane
    constexpr int VJ = (V + J - 1) / J;                        // chain j: vectors [j*VJ, ...)
    extern __shared__ __align__(16) int ms_smem[];            // [S][NW][SEG]
    __shared__ __align__(8) uint64_t bars[S][NW];
    __shared__ MsTup red[NW];
    __shared__ bool am_last;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) DC_MS_TRACE_AT(blockIdx.x * 16 + 0);

    // this warp's range [wbeg, wend) (RW is a multiple of SEG); CTA-local indices
    const long long cbase = min(n, (long long)blockIdx.x * NW * RW);
    const long long wbeg = min(n, ((long long)blockIdx.x * NW + warp) * RW);
    const long long wend = min(n, wbeg + RW);
    const int nseg = (int)((wend - wbeg + SEG - 1) / SEG);

    if (lane == 0) {
#pragma unroll
        for (int s = 0; s < S; ++s) mbar_init(smem_addr(&bars[s][warp]), 1);
    }
    __syncwarp();
    auto seg_ptr = [&](int s) { return ms_smem + (s * NW + warp) * SEG; };
    auto issue = [&](int k) {          // lane 0: segment k -> stage k % S
        const int s = k % S;
        const uint32_t bar = smem_addr(&bars[s][warp]);
        const long long g0 = wbeg + (long long)k * SEG;
        const int cnt = (int)min((long long)SEG, wend - g0);
        const int body = cnt & ~3;    // 16-byte part (g0 is 16-byte aligned)
        mbar_arrive_expect_tx(bar, 4u * body);
        if (body) bulk_g2s(smem_addr(seg_ptr(s)), x + g0, 4u * body, bar);
    };
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < S; ++k)
            if (k < nseg) issue(k);
    }

    MsFold acc;                        // lane 0: the warp's running summary
    acc.init();
    for (int k = 0; k < nseg; ++k) {
        const int s = k % S;
        mbar_wait(smem_addr(&bars[s][warp]), (uint32_t)((k / S) & 1));
        const long long g0 = wbeg + (long long)k * SEG;
        const int cnt = (int)min((long long)SEG, wend - g0);
        const int* sl = seg_ptr(s) + lane * L;
        const int e0 = lane * L;                     // first element of this lane
        const int i0 = (int)(g0 - cbase) + e0;
        MsFold f;
        f.init();
        if (VO) {
            MsVal v;
            v.init();
            if (cnt == SEG) {
                MsVal g[J];
#pragma unroll
                for (int j = 0; j < J; ++j) g[j].init();
#pragma unroll
                for (int q = 0; q < VJ; ++q) {
#pragma unroll
                    for (int j = 0; j < J; ++j) {
                        if (j * VJ + q < V && q < VJ) {
                            const int4 w = *reinterpret_cast<const int4*>(sl + 4 * (j * VJ + q));
                            g[j].step(w.x);
                            g[j].step(w.y);
                            g[j].step(w.z);
                            g[j].step(w.w);
                        }
                    }
                }
#pragma unroll
                for (int j = 0; j < J; ++j) v.absorb(g[j]);
            } else {
                const int body = cnt & ~3;
                for (int e = e0; e < min(cnt, e0 + L); ++e)
                    v.step(e < body ? sl[e - e0] : x[g0 + e]);
            }
            // one leaf per lane chunk, labelled by its start (an empty chunk
            // keeps the identity's sentinels and is absorbed without effect)
            f.tot = v.tot; f.pre = v.pre; f.suf = v.suf; f.best = v.best;
            f.pe = f.ss = f.bs = f.be = i0;
        } else if (cnt == SEG) {
            MsFold g[J];
#pragma unroll
            for (int j = 0; j < J; ++j) g[j].init();
#pragma unroll
            for (int q = 0; q < VJ; ++q) {
#pragma unroll
                for (int j = 0; j < J; ++j) {
                    if (j * VJ + q < V && q < VJ) {          // compile-time after unrolling
                        const int o = 4 * (j * VJ + q);
                        const int4 v = *reinterpret_cast<const int4*>(sl + o);
                        g[j].step(v.x, i0 + o);
                        g[j].step(v.y, i0 + o + 1);
                        g[j].step(v.z, i0 + o + 2);
                        g[j].step(v.w, i0 + o + 3);
                    }
                }
            }
#pragma unroll
            for (int j = 0; j < J; ++j) f.absorb(g[j]);
        } else {                                     // the warp's last, partial segment
            const int body = cnt & ~3;
            for (int e = e0; e < min(cnt, e0 + L); ++e)
                f.step(e < body ? sl[e - e0] : x[g0 + e], i0 + (e - e0));
        }
        __syncwarp();                                // reconverge before the shuffle tree
        f = ms_fold_warp(f);
        if (lane == 0) acc.absorb(f);
        __syncwarp();                                // every lane is done with stage s
        if (lane == 0 && k + S < nseg) {
            fence_proxy_async_smem();
            issue(k + S);
        }
    }

    // ---- warps -> CTA summary: an ordered branch-free tree over the NW warp
    // summaries in warp 0; the part is published with a release atomic on the
    // ticket (acq_rel: the last CTA also acquires every other part)
    if (lane == 0) red[warp] = acc.tup();
    if (lane == 0) DC_MS_TRACE_AT(blockIdx.x * 16 + 1 + warp);
    __syncthreads();
    if (warp == 0) {
        MsTupG c = lane < NW ? ms_widen(red[lane], cbase) : ms_empty<long long>();
        c = ms_warp_combine<NW>(c);
        if (lane == 0) {
            ms_store(&parts[blockIdx.x], c, 0);
            unsigned int prev;
            asm volatile("atom.add.acq_rel.gpu.u32 %0, [%1], 1;" : "=r"(prev) : "l"(ticket) : "memory");
            am_last = prev == gridDim.x - 1;
        }
    }
    __syncthreads();
    if (tid == 0) DC_MS_TRACE_AT(blockIdx.x * 16 + 15);
    if (!am_last || warp != 0) return;         // (lane 0's acq_rel ticket + the barrier order the loads below)

    // ---- NK5 (warp 0 of the last CTA): lane l folds the contiguous parts
    // [l*per, (l+1)*per) (loads issued together), then one ordered warp tree
    const int np = gridDim.x;
    const int per = (np + 31) / 32;
    MsTupG a = ms_empty<long long>();
    constexpr int kPer = 5;                    // parts loaded at once per lane (148 SMs: one round)
    for (int q0 = 0; q0 < per; q0 += kPer) {
        MsTupG v[kPer];
#pragma unroll
        for (int q = 0; q < kPer; ++q) {
            const int i = lane * per + q0 + q;
            v[q] = (q0 + q < per && i < np) ? ms_load_cg(parts + i) : ms_empty<long long>();
        }
#pragma unroll
        for (int q = 0; q < kPer; ++q) a = ms_combine(a, v[q]);
    }
    a = ms_warp_combine<32>(a);
    a.tot = __shfl_sync(0xffffffffu, a.tot, 0);
    a.pre = __shfl_sync(0xffffffffu, a.pre, 0);
    a.suf = __shfl_sync(0xffffffffu, a.suf, 0);
    a.best = __shfl_sync(0xffffffffu, a.best, 0);
    a.pe = __shfl_sync(0xffffffffu, a.pe, 0);
    a.ss = __shfl_sync(0xffffffffu, a.ss, 0);
    a.bs = __shfl_sync(0xffffffffu, a.bs, 0);
    a.be = __shfl_sync(0xffffffffu, a.be, 0);
    if (VO) ms_recover<L>(x, n, a, nullptr);
    if (tid == 0) {
        if (mode == 0) {
            out_res->sum = a.best;
            out_res->start = a.bs + off;
            out_res->end = a.be + off;
        } else {
            ms_store(out_tup, a, off);
        }
        *ticket = 0u;
        DC_MS_TRACE_AT(2047 * 16);
    }
}

}  // namespace dc
