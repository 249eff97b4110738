// sort4_kernels.cuh -- two levels of the merge tree per HBM pass.
//
// A pass over runs of width w merges every group of four adjacent runs
// (R0 R1 R2 R3) into one run of 4w: merge(merge(R0, R1), merge(R2, R3)),
// i.e. Alg 7's combine applied at two consecutive levels of the
// binary tree, the intermediate runs living only in shared memory.  Every
// merge is the stable one of the one-level pass (earlier run wins ties), so
// the output order is the composite order (key, run, position) and the result
// is bit-identical to two one-level passes; only the HBM traffic halves.
//
//   NK2-4 select : for every output tile boundary of a group, the exact cut
//                  (c0, c1, c2, c3), c_q = #R_q elements among the first d
//                  outputs -- a warp-parallel multi-sequence selection that
//                  brackets 8 pivots per run every round (one dependent load
//                  per round instead of a nested binary search);
//   NK3-4 merge  : persistent CTAs, double-buffered: the four pieces of the
//                  next tile arrive by TMA while the current tile is merged
//                  (stage 1: piece pairs -> X, Y in registers; stage 2: X with
//                  Y in a bitonic layout), the tile leaves by a TMA bulk store.
//
// Tiles: every group is cut into tpg = ceil(min(4w, n) / T) output tiles of T
// keys (the last one of a group short, trailing ones of the last group
// empty); tile j is local tile j % tpg of group j / tpg.  Positions inside a
// group fit in int32 (n < 2^31).
//
// The same kernels merge ONE group of four runs of arbitrary lengths that
// live in separate buffers (Pass4 custom mode): the local G-way merge of the
// multi-GPU sort (a9, Alg 7's top levels) reads up to four received runs --
// or four peer GPUs' sorted shards over NVLink, the exchange fused into the
// merge -- and writes their stable merge in one HBM pass.
//
// Keys-only (u32 / i32): equal keys are identical bit patterns, so the merges
// use +inf pads instead of bounds checks (see merge_pad).
#pragma once
#include <cstdint>

namespace dc {

struct Cut4 {
    int c[4];
};

// The runs of one two-level pass.
//   uniform (custom == 0): groups of four adjacent runs of width w over
//     [0, n) of one buffer (k[q] = src, v[q] = src values, bound[q] = n);
//   custom  (custom == 1): ONE group; run q is len[q] elements at offset
//     off[q] of buffer k[q] (+ v[q]), readable for bound[q] elements, and the
//     merged group goes to dst[out0, out0 + sum len).
// Buffer bases are 16-byte aligned (TMA); they may be peer-GPU mappings.
struct Pass4 {
    const uint32_t* k[4];
    const uint32_t* v[4];
    long long bound[4];
    long long off[4];
    long long len[4];
    long long n, w, out0;
    int T, tpg, custom;
};

// Tile j of a pass: the start of each run in its buffer, the four run
// lengths, the group length, the group's output offset o and the tile's
// output range [d0, d1) relative to o (empty when d0 >= tot, in the last
// group of a uniform pass).
struct Tile4Geo {
    long long st[4];
    long long o;
    int l[4];
    int tot, d0, d1;
    __device__ __forceinline__ Tile4Geo(const Pass4& P, int j) {
        const int G = P.custom ? 0 : j / P.tpg;
        tot = 0;
        if (P.custom) {
            o = P.out0;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                st[q] = P.off[q];
                l[q] = (int)P.len[q];
                tot += l[q];
            }
        } else {
            o = (long long)G * 4 * P.w;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                st[q] = o + q * P.w;
                l[q] = (int)max(0LL, min(P.w, P.n - o - q * P.w));
                tot += l[q];
            }
        }
        const long long e0 = (long long)(j - G * P.tpg) * P.T;   // may pass tot (empty tile)
        d0 = (int)min(e0, (long long)tot);
        d1 = (int)min(e0 + P.T, (long long)tot);
    }
};

// Composite order of the 4-way stable merge: element x of run qx precedes
// element e of run qe iff x < e, or x == e and qx < qe (same run: position).
template <class K>
__device__ __forceinline__ bool precedes(uint32_t x, int qx, uint32_t e, int qe) {
    return K::lt(x, e) | ((!K::lt(e, x)) & (qx < qe));
}

// Position of pivot t (0..PV-1) in a window [lo, lo + W): evenly spaced when
// W >= PV + 1 (strictly inside the window), every position when W <= PV.
template <int PV>
__device__ __forceinline__ int sel4_pivot(int lo, int W, int step, int t) {
    return lo + (W >= PV + 1 ? (t + 1) * step : min(t, W - 1));
}

// ------------------------------------------------------------------ NK2-4
#ifndef DC_SEL4_EXACT_FROM
#define DC_SEL4_EXACT_FROM 48
#endif
// A group of LB = 4*PV lanes per tile boundary (PV = 8: one boundary per
// warp; PV = 4: two).  Lane l of a group owns pivot t = l % PV of run
// q = l / PV.  Invariant: lo_q <= c_q <= hi_q, with the values R_q[lo_q - 1]
// (taken) and R_q[hi_q] (not taken) known.  Every round each run with a
// non-empty window puts PV pivots in it; a pivot E (run q, position p) is
//   * taken      if it precedes a known taken edge of another run, or if
//                 p + sum_q' U_q'(E) < d,
//   * not taken  if a known untaken edge precedes it, or p + sum L_q'(E) >= d,
// where [L_q', U_q'] brackets #R_q' elements preceding E between the
// neighbouring pivots of run q' (positions in closed form, values by
// shuffle).  The largest taken pivot raises lo_q, the smallest untaken one
// lowers hi_q.  Once every window has <= PV elements all of them are pivots,
// the brackets are exact and every window closes: c_q = lo_q.
// The cut of tile j's first output, computed by a converged warp (valid in
// every lane of the boundary's group).  An empty tile (end of the last
// group) or !valid gets the zero cut; its lanes still take part in the
// warp's shuffles until every group of the warp is done.
template <class K, int PV = 8>
__device__ __forceinline__ Cut4 select4_warp(const Pass4& P, int j, bool valid = true) {
    static_assert(PV == 8 || PV == 4 || PV == 2, "8, 4 or 2 pivots per run (1, 2, 4 boundaries per warp)");
    constexpr int LB = 4 * PV;
    const int lane = threadIdx.x & 31;
    const int base = lane & ~(LB - 1);                 // first lane of this boundary's group
    const int ll = lane - base;
    const int q = ll / PV, t = ll % PV;
    const Tile4Geo g(P, valid ? j : 0);
    const int d = g.d0;
    const bool live = valid && d < g.tot;
    if (PV == 8 && !live) return Cut4{{0, 0, 0, 0}}; // whole warp: uniform exit
    const uint32_t* R[4];
#pragma unroll
    for (int r = 0; r < 4; ++r) R[r] = P.k[r] + g.st[r];
    const uint32_t* Rq = R[0];
#pragma unroll
    for (int r = 1; r < 4; ++r)
        if (q == r) Rq = R[r];
    int lo[4], hi[4];
    uint32_t elo[4], ehi[4];
    {
        // initial windows and their edge values (group lane r: R_r[lo_r - 1],
        // group lane 4+r: R_r[hi_r]); a dead group has every window closed
        uint32_t ev = 0;
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            lo[r] = live ? max(0, d - (g.tot - g.l[r])) : 0;
            hi[r] = live ? min(g.l[r], d) : 0;
            const int pos = ll == r ? lo[r] - 1 : hi[r];
            if (live && (ll == r || ll == 4 + r) && pos >= 0 && pos < g.l[r])
                ev = __ldg(R[r] + pos);
        }
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            elo[r] = __shfl_sync(0xffffffffu, ev, base + r);
            ehi[r] = __shfl_sync(0xffffffffu, ev, base + 4 + r);
        }
    }
#ifdef DC_SEL4_MAXROUNDS
    int dbg_rounds = 0;
#endif
    // One round; false once every window of every group in the warp is
    // closed.  Progress guard: from round DC_SEL4_EXACT_FROM on (the EXACT
    // instantiation, a separate loop so the common rounds carry no fallback
    // code), every undecided pivot's brackets are resolved by exact binary
    // searches, so every round decides every pivot (never reached on the
    // tested inputs).
    auto round_step = [&](auto exact_tag) -> bool {
        constexpr bool exact = decltype(exact_tag)::value;
#ifdef DC_SEL4_MAXROUNDS
        if (++dbg_rounds > DC_SEL4_MAXROUNDS) {
            if (ll == 0) printf("select4 stall j=%d d=%d\n", j, d);
            return false;
        }
#endif
        int W[4], st[4], open = 0;
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            W[r] = hi[r] - lo[r];
            st[r] = W[r] / (PV + 1);
            open |= W[r];
        }
        if (PV == 8) {
            if (open == 0) return false;
        } else if (!__any_sync(0xffffffffu, open != 0)) {
            return false;
        }
        int Wq = W[0], loq = lo[0], stq = st[0];
#pragma unroll
        for (int r = 1; r < 4; ++r)
            if (q == r) { Wq = W[r]; loq = lo[r]; stq = st[r]; }
        const bool active = Wq > 0;
        const int p = sel4_pivot<PV>(loq, Wq, stq, t);
        const uint32_t v = active ? __ldg(Rq + p) : 0u;
        int SL = p, SU = p;
        bool dt = false, du = false;
        // (every shuffle below runs unconditionally on the converged warp; the
        //  own run and closed windows are masked with selects)
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            // #pivots of run r preceding this lane's pivot (search over the group's lanes PV*r ..)
            int a = 0;                                   // in [0, PV]
#pragma unroll
            for (int step = PV / 2; step >= 1; step >>= 1) {
                const uint32_t V = __shfl_sync(0xffffffffu, v, base + PV * r + a + step - 1);
                a += precedes<K>(V, r, v, q) ? step : 0;
            }
            const uint32_t VL = __shfl_sync(0xffffffffu, v, base + PV * r + PV - 1);
            a += (a == PV - 1 && precedes<K>(VL, r, v, q)) ? 1 : 0;
            const bool other = r != q;
            dt |= other & (lo[r] > 0) & !precedes<K>(elo[r], r, v, q);      // E before a taken edge
            du |= other & (hi[r] < g.l[r]) & precedes<K>(ehi[r], r, v, q);  // untaken edge before E
            // (branch-free: the positions of pivots a-1 and a of run r)
            const bool big = W[r] >= PV + 1;
            const int pa1 = lo[r] + (big ? a * st[r] : min(a - 1, W[r] - 1));
            const int pa = lo[r] + (big ? (a + 1) * st[r] : min(a, W[r] - 1));
            int Lp = (W[r] > 0) & (a > 0) ? pa1 + 1 : lo[r];
            int Up = (W[r] > 0) & (a < PV) ? pa : hi[r];
            if constexpr (exact) {
                if (other && !(dt | du) && active) {
                    int x0 = Lp, x1 = Up;                // first position not preceding E
                    while (x0 < x1) {
                        const int mid = (x0 + x1) >> 1;
                        if (precedes<K>(__ldg(R[r] + mid), r, v, q)) x0 = mid + 1;
                        else x1 = mid;
                    }
                    Lp = Up = x0;
                }
            }
            SL += other ? Lp : 0;
            SU += other ? Up : 0;
        }
        // The brackets hold only for a pivot between every other run's edges;
        // an edge decision takes precedence (dt and du exclude each other).
        const bool taken = active && (dt || (!du && SU < d));
        const bool untaken = active && (du || (!dt && SL >= d));
        const unsigned mt = __ballot_sync(0xffffffffu, taken) >> base;
        const unsigned mu = __ballot_sync(0xffffffffu, untaken) >> base;
        constexpr unsigned PM = (1u << PV) - 1u;
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            const unsigned gt = (mt >> (PV * r)) & PM, gu = (mu >> (PV * r)) & PM;
            const int tt = 31 - __clz(gt | 1u);             // largest taken pivot (0 if none)
            const int tu = __ffs(gu | (1u << (PV - 1))) - 1;   // smallest untaken (PV-1 if none)
            const uint32_t vt = __shfl_sync(0xffffffffu, v, base + PV * r + tt);
            const uint32_t vu = __shfl_sync(0xffffffffu, v, base + PV * r + tu);
            const int lo0 = lo[r];                          // this round's pivot base
            const int nlo = sel4_pivot<PV>(lo0, W[r], st[r], tt) + 1;
            const int nhi = sel4_pivot<PV>(lo0, W[r], st[r], tu);
            elo[r] = gt ? vt : elo[r];                      // (branch-free updates)
            lo[r] = gt ? nlo : lo[r];
            ehi[r] = gu ? vu : ehi[r];
            hi[r] = gu ? nhi : hi[r];
        }
        return true;
    };
    int round = 0;
    bool more = true;
    for (; more && round < DC_SEL4_EXACT_FROM; ++round) more = round_step(std::false_type{});
    for (; more; ++round) more = round_step(std::true_type{});
#ifdef DC_SEL4_ROUNDS_OUT   // measurement hook (tools/select4_rounds.cu): rounds per boundary
    if (valid && ll == 0) DC_SEL4_ROUNDS_OUT[j] = round;
#endif
    Cut4 c;
#pragma unroll
    for (int r = 0; r < 4; ++r) c.c[r] = lo[r];
    return c;
}

// NK2-4 as its own launch: BPW = 32 / (4 PV) tile boundaries per warp.
// Measured at 2^28: keys-only PV 8 / 4 / 2 -> 0.472 / 0.443 / 0.396 ms per
// sort; key-value (twice the tiles) 0.818 / 0.698 / 0.709 ms.
template <int PV>
constexpr int sel4_bpw() { return 32 / (4 * PV); }
template <class K, int PV>
__global__ void nk2_select4(const Pass4 P, int num_tiles, Cut4* __restrict__ cut) {
    constexpr int LB = 4 * PV, BPW = 32 / LB;
    const int wj = (int)(((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * BPW;
    if (wj >= num_tiles) return;                      // warp-uniform
    const int lane = threadIdx.x & 31;
    const int j = wj + lane / LB;
    const bool valid = j < num_tiles;
    const Cut4 c = select4_warp<K, PV>(P, j, valid);
    if (valid && lane % LB == 0) {
        const Tile4Geo g(P, j);
        if (g.d0 < g.tot) cut[j] = c;                 // (empty tiles: no cut)
    }
}

// ------------------------------------------------------------------ NK3-4
// Pad-safe serial merge of IT outputs (keys only): each piece in shared memory
// is followed by >= IT pads of K::kPad (the maximum key).  "take B iff b < a"
// then never needs a bound: an exhausted side reads pads, which lose against
// every smaller key, and against an equal (maximum) key the pad is emitted in
// its place -- the same bit pattern, and only maximum keys remain.
template <class K, int IT>
__device__ __forceinline__ void merge_pad(uint32_t ai, uint32_t bi, uint32_t (&out)[IT]) {
    uint32_t a = lds(ai), b = lds(bi);
    const uint32_t c0 = ai + bi;
#pragma unroll
    for (int j = 0; j < IT; ++j) {
        const bool p = K::lt(b, a);
        out[j] = p ? b : a;
        if (!p) ai += 4u;
        bi = c0 + 4u * (j + 1) - ai;
        const uint32_t v = lds(p ? bi : ai);
        if (p) b = v; else a = v;
    }
}

// Per-buffer tile descriptor, written by the producer.
struct Tile4 {
    long long g0[4];  // global start of each piece
    int len[4];
    int at[4];        // word offset of each piece's first element in the region
    long long out;    // global output offset of the tile
    int total;
    int pad_;
};

// Shared words of one key (or value) region of a buffer: a guard of IT + 4
// words (the bitonic stage-2 merge of a short tile may read just below the
// region), then the four pieces with their alignment heads and IT pads each.
// A buffer is one key region (keys only) or a key region followed by a value
// region with the same layout; there are two buffers.
__host__ __device__ constexpr int m4_guard(int IT) { return (IT + 4 + 3) / 4 * 4; }
__host__ __device__ constexpr int m4_region_words(int T, int IT) {
    return m4_guard(IT) + (T + 4 * (IT + 8) + 16 + 3) / 4 * 4;
}
__host__ __device__ constexpr int m4_smem_bytes(int T, int IT, bool vals) {
    return 2 * (vals ? 2 : 1) * m4_region_words(T, IT) * 4;
}

__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
// Barrier among the NC consumer threads only (named barrier 1).
template <int NC>
__device__ __forceinline__ void consumer_sync() {
    asm volatile("bar.sync 1, %0;" ::"n"(NC) : "memory");
}

// NK3-4: persistent 4-way tile merge, warp-specialised and double-buffered.
// NT + 64 threads.  Consumers (threads 0..NT+31): stage 1 needs up to NT + 1
// windows of IT outputs (X and Y windowed separately), stage 2 uses NT
// threads.  Producer (the last warp): fills a buffer with a tile (pads and
// ragged piece ends by plain stores, the 16-byte-aligned interior of every
// piece by TMA), and once the consumers have written a tile's output back
// into its buffer, bulk-stores it and refills the buffer with the tile two
// ahead.  full[b]: tile data present (producer arrive + TMA bytes);
// empty[b]: output written (one arrive per consumer warp).  Tiles
// J = blockIdx.x + i * gridDim.x; empty tiles (end of the last group) pass
// through with no work.  (An in-kernel selection -- selector warps filling a
// cut ring ahead of the producer -- was measured slower than the separate
// NK2-4 launch and removed.)
//
// Keys-only u32/i32 (equal keys indistinguishable): pad-safe merges and a
// bitonic stage 2 (Y stored descending), no bounds checks.  Stable variants
// (values, or f32 keys whose +0/-0 must keep their order): bounds-checked
// stable merges (earlier run wins ties: R0 < R1 within X, R2 < R3 within Y,
// X < Y), values gathered through the source address of every key.
#ifndef DC_M4_MINB   // CTAs per SM the register budget is sized for
#define DC_M4_MINB 1
#endif
// Sanitizer variant (-DDC_M4_BARRIER_HANDOFF, tools/sanitize.sh only): the same
// kernel with every producer/consumer hand-off done by named barriers
// (bar.arrive / bar.sync, which compute-sanitizer racecheck models) instead of
// mbarriers, and the pieces and outputs moved by plain loads and stores
// instead of TMA.  The merge code is unchanged; racecheck runs clean on it,
// which isolates the default build's reports to the mbarrier/TMA hand-off.
#ifndef DC_M4_BARRIER_HANDOFF
#define DC_M4_BARRIER_HANDOFF 0
#endif
template <int NC>
__device__ __forceinline__ void named_arrive(int id) {
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "n"(NC + 32) : "memory");
}
template <int NC>
__device__ __forceinline__ void named_sync(int id) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "n"(NC + 32) : "memory");
}
template <int NT, int IT, class K, bool V>
__global__ void __launch_bounds__(NT + 64, DC_M4_MINB)
nk3_merge4(const Pass4 P, uint32_t* __restrict__ dst_k, uint32_t* __restrict__ dst_v,
           const Cut4* __restrict__ cut, int num_tiles) {
    static_assert(IT % 2 == 1, "odd items per thread keep the blocked layout conflict-free");
    constexpr bool kStable = V || K::kNeedStable;
    constexpr int T = NT * IT;
    constexpr int NC = NT + 32;                        // consumer threads
    constexpr int KW = m4_region_words(T, IT);
    constexpr int BW = (V ? 2 : 1) * KW;               // words per buffer
    constexpr int GU = m4_guard(IT);
    constexpr uint32_t VOFF = 4u * KW;                 // key -> value byte offset
    extern __shared__ __align__(16) uint32_t sm[];
    __shared__ __align__(8) uint64_t full[2], empty[2];
    __shared__ Tile4 meta[2];
    const int tid = threadIdx.x;
    const int lane = tid & 31;
    const uint32_t SM0 = smem_addr(sm);
    const int my_tiles = (int)blockIdx.x < num_tiles
                             ? (num_tiles - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 0;
    auto tile_of = [&](int i) { return (int)blockIdx.x + i * (int)gridDim.x; };

    if (tid == 0) {
#pragma unroll
        for (int b = 0; b < 2; ++b) {
            mbar_init(smem_addr(&full[b]), 1);
            mbar_init(smem_addr(&empty[b]), NC / 32);
        }
    }
    __syncthreads();

    if (tid >= NC) {
        // ------------------------------------------------------ producer warp
        // Fill buffer b with tile J: cut vectors (start; end = next tile's
        // start or the run lengths at the end of a group) -> pieces.  The TMA
        // copies each piece's 16-byte-aligned interior [g0 & ~3, tend) from its
        // run's buffer; the lanes store the ragged end (< 4 words, or the part
        // at/after the buffer's aligned bound) and IT pads behind each piece.
        auto fill = [&](int i, int b) {
            const int J = tile_of(i);
            const Tile4Geo g(P, J);
            int c0[4], c1[4];
            if (g.d0 < g.tot) {
                const Cut4 a = cut[J];
                Cut4 e;
                if (g.d1 == g.tot) {
#pragma unroll
                    for (int r = 0; r < 4; ++r) e.c[r] = g.l[r];
                } else {
                    e = cut[J + 1];
                }
#pragma unroll
                for (int r = 0; r < 4; ++r) { c0[r] = a.c[r]; c1[r] = e.c[r]; }
            } else {
#pragma unroll
                for (int r = 0; r < 4; ++r) c0[r] = c1[r] = 0;
            }
            Tile4 m;
            m.out = g.o + g.d0;
            m.total = max(0, g.d1 - g.d0);
            uint32_t* buf = sm + b * BW + GU;
            const uint32_t base = SM0 + 4u * (b * BW + GU);
            uint32_t bytes = 0;
            long long tend[4];
            int o = 0;
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                const uint32_t* rk = P.k[r];
                m.g0[r] = g.st[r] + c0[r];
                m.len[r] = c1[r] - c0[r];
                m.at[r] = o + (int)(m.g0[r] & 3);
                const long long n4 = P.bound[r] & ~3LL;
                const long long al0 = m.g0[r] & ~3LL;
                long long al1 = (m.g0[r] + m.len[r]) & ~3LL;
                if (al1 > n4) al1 = n4;
                if (al1 < al0 || DC_M4_BARRIER_HANDOFF) al1 = al0;   // (variant: all plain loads)
                tend[r] = al1;
                if (al1 > al0) bytes += (uint32_t)(4 * (al1 - al0)) * (V ? 2 : 1);
                o = (m.at[r] + m.len[r] + IT + 1 + 3) & ~3;
                const int e0 = (int)(max(al1, m.g0[r]) - m.g0[r]);
                for (int e = e0 + lane; e < m.len[r] + IT; e += 32) {
                    const bool real = e < m.len[r];
                    buf[m.at[r] + e] = real ? rk[m.g0[r] + e] : K::kPad;
                    if (V) buf[KW + m.at[r] + e] = real ? P.v[r][m.g0[r] + e] : 0u;
                }
            }
            __syncwarp();
            if (DC_M4_BARRIER_HANDOFF) {
                if (lane == 0) meta[b] = m;
                named_arrive<NC>(2 + b);                 // full[b]
                return;
            }
            if (lane == 0) {
                meta[b] = m;
                const uint32_t fb = smem_addr(&full[b]);
                mbar_arrive_expect_tx(fb, bytes);        // release: pads + meta
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    const long long al0 = m.g0[r] & ~3LL;
                    if (tend[r] > al0) {
                        const uint32_t d = base + 4u * (m.at[r] - (int)(m.g0[r] & 3));
                        const uint32_t nb = (uint32_t)(4 * (tend[r] - al0));
                        bulk_g2s(d, P.k[r] + al0, nb, fb);
                        if (V) bulk_g2s(d + VOFF, P.v[r] + al0, nb, fb);
                    }
                }
            }
        };
        if (my_tiles > 0) fill(0, 0);
        if (my_tiles > 1) fill(1, 1);
        for (int i = 0; i < my_tiles; ++i) {
            const int b = i & 1;
            if (DC_M4_BARRIER_HANDOFF) {
                named_sync<NC>(4 + b);                   // empty[b]: output of tile i written
                const Tile4 m = meta[b];
                const int h = (int)(m.out & 3);
                const int head = min(m.total, (4 - h) & 3);
                const int body = (m.total - head) & ~3;
                const uint32_t* ob = sm + b * BW + GU + h;
                for (int e = head + lane; e < head + body; e += 32) {
                    dst_k[m.out + e] = ob[e];
                    if (V) dst_v[m.out + e] = ob[KW + e];
                }
                __syncwarp();
                if (i + 2 < my_tiles) fill(i + 2, b);
                continue;
            }
            mbar_wait(smem_addr(&empty[b]), (i >> 1) & 1);   // output of tile i written
            if (lane == 0) {
                const Tile4 m = meta[b];
                // output element e sits at buffer word h + e (h = m.out mod 4),
                // so the 16-byte-aligned body [head, head + body) is aligned on
                // both sides of the bulk store; head and tail left by plain stores
                const int h = (int)(m.out & 3);
                const int head = min(m.total, (4 - h) & 3);
                const int body = (m.total - head) & ~3;
                if (body > 0) {
                    const uint32_t sb = SM0 + 4u * (b * BW + GU + h + head);
                    bulk_s2g(dst_k + m.out + head, sb, 4u * body);
                    if (V) bulk_s2g(dst_v + m.out + head, sb + VOFF, 4u * body);
                    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                }
                if (i + 2 < my_tiles) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            }
            __syncwarp();
            if (i + 2 < my_tiles) fill(i + 2, b);
        }
        if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
        return;
    }

    // ---------------------------------------------------------- consumers
// Stage-2 co-ranks seeded by one 32-ary warp search per warp (each lane then
// searches [c(D), c(D) + lane*IT] only).  Measured r02b at 2^28 u32: merges
// 3.761 vs 3.702 ms per sort (the warp rounds cost more issue slots than the
// ~5 binary steps per lane they save; profiles/r02b/m4_warp_corank.txt): off.
#ifndef DC_M4_WARP_CORANK
#define DC_M4_WARP_CORANK 0
#endif
#ifndef DC_M4_SKIP   // measurement knob: bit 0 skips stage 1, bit 1 stage 2
#define DC_M4_SKIP 0
#endif
    for (int i = 0; i < my_tiles; ++i) {
        const int b = i & 1;
        uint32_t* buf = sm + b * BW + GU;
        const uint32_t B0 = SM0 + 4u * (b * BW + GU);
        if (DC_M4_BARRIER_HANDOFF) named_sync<NC>(2 + b);
        else mbar_wait(smem_addr(&full[b]), (i >> 1) & 1);
        const Tile4 m = meta[b];

        // stage 1: X = merge(P0, P1), Y = merge(P2, P3), IT-output windows
        const int nx = m.len[0] + m.len[1], ny = m.len[2] + m.len[3];
        const int total = nx + ny;
        const int wx = (nx + IT - 1) / IT, wy = (ny + IT - 1) / IT;
        uint32_t k[IT], src[IT], vv[IT];
        int valid = 0, base_out = 0;
        bool up = true;
        if (!(DC_M4_SKIP & 1) && tid < wx + wy) {
            const bool first = tid < wx;
            const int na = first ? m.len[0] : m.len[2], nb = first ? m.len[1] : m.len[3];
            const uint32_t A = B0 + 4u * (first ? m.at[0] : m.at[2]);
            const uint32_t Bq = B0 + 4u * (first ? m.at[1] : m.at[3]);
            const int diag = (first ? tid : tid - wx) * IT;
            const int ci = corank_smem<K>(A, na, Bq, nb, diag);
            if constexpr (kStable) {
                serial_merge<K, IT, V>(A + 4u * ci, A + 4u * na, Bq + 4u * (diag - ci),
                                       Bq + 4u * nb, k, src);
                if (V) {
#pragma unroll
                    for (int q = 0; q < IT; ++q) vv[q] = lds(src[q] + VOFF);
                }
                // X at [0, nx), Y at [nx, nx + ny), both ascending
                base_out = first ? diag : nx + diag;
            } else {
                merge_pad<K, IT>(A + 4u * ci, Bq + 4u * (diag - ci), k);
                // X ascending at [0, nx); Y descending at [nx, nx + ny)
                up = first;
                base_out = first ? diag : nx + ny - 1 - diag;
            }
            valid = min(IT, na + nb - diag);
        }
        consumer_sync<NC>();                           // all pieces consumed
        if (valid == IT) {                             // full window: unconditional stores
            uint32_t* o = buf + base_out;
            if (up) {
#pragma unroll
                for (int q = 0; q < IT; ++q) {
                    o[q] = k[q];
                    if (V) o[KW + q] = vv[q];
                }
            } else {
#pragma unroll
                for (int q = 0; q < IT; ++q) o[-q] = k[q];
            }
        } else {
#pragma unroll
            for (int q = 0; q < IT; ++q)
                if (q < valid) {
                    const int at = up ? base_out + q : base_out - q;
                    buf[at] = k[q];
                    if (V) buf[KW + at] = vv[q];
                }
        }
        consumer_sync<NC>();

        const int diag = tid * IT;
        const bool act2 = tid < NT && diag < total;
        if (act2 && !(DC_M4_SKIP & 2)) {
            if constexpr (kStable) {
                // stage 2: stable merge of X and Y (X wins ties)
                const int c = corank_smem<K>(B0, nx, B0 + 4u * nx, ny, diag);
                serial_merge<K, IT, V>(B0 + 4u * c, B0 + 4u * nx, B0 + 4u * (nx + diag - c),
                                       B0 + 4u * total, k, src);
                if (V) {
#pragma unroll
                    for (int q = 0; q < IT; ++q) vv[q] = lds(src[q] + VOFF);
                }
            } else {
                // stage 2: bitonic merge of X (ascending) and Y (descending)
                const uint32_t Ab = B0, Bb = B0 + 4u * (total - diag);
                int lo = max(0, diag - ny), hi = min(diag, nx);
#if DC_M4_WARP_CORANK
                if (__activemask() == 0xffffffffu) {   // (the tile's last warp may be partial)
                    // The warp's lanes own consecutive diagonals D + l*IT, so
                    // c(D + l*IT) lies in [c(D), c(D) + l*IT].  c(D) by a 32-ary
                    // warp search (probes spread over the window, ~3 rounds),
                    // then every lane's binary search starts from that window.
                    const int D = diag - lane * IT;
                    int wlo = max(0, D - ny), whi = min(D, nx);
                    const uint32_t Bd = B0 + 4u * (total - D);
                    while (whi > wlo) {
                        const int step = (whi - wlo + 31) >> 5;
                        const int q = wlo + (lane + 1) * step - 1;   // P(q): q < c(D)
                        const bool ok = q < whi && !K::lt(lds(Bd + 4u * q), lds(Ab + 4u * q));
                        const int nt = __popc(__ballot_sync(0xffffffffu, ok));
                        const int nlo = wlo + nt * step;
                        whi = min(whi, wlo + (nt + 1) * step - 1);
                        wlo = nlo;
                    }
                    lo = max(lo, wlo);
                    hi = min(hi, wlo + lane * IT);
                }
#endif
                while (lo < hi) {
                    const int mid = (lo + hi) >> 1;
                    if (!K::lt(lds(Bb + 4u * mid), lds(Ab + 4u * mid))) lo = mid + 1;
                    else hi = mid;
                }
                uint32_t ai = Ab + 4u * lo;
                const uint32_t bi0 = B0 + 4u * (total - 1 - (diag - lo));
                const uint32_t D = ai - bi0;
                uint32_t a = lds(ai), bv = lds(bi0);
#pragma unroll
                for (int q = 0; q < IT; ++q) {
                    const bool p = K::lt(bv, a);
                    k[q] = p ? bv : a;
                    if (!p) ai += 4u;
                    const uint32_t bi = ai - D - 4u * (q + 1);
                    const uint32_t v = lds(p ? bi : ai);
                    if (p) bv = v; else a = v;
                }
            }
        }
        consumer_sync<NC>();
        // output back into the buffer at word h + e (the producer bulk-stores
        // the 16-byte-aligned body); the < 4-word head (custom passes may
        // start anywhere) and tail straight from registers.  Uniform passes
        // start at multiples of 4 words (T and 4w are): h = head = 0.
        const int h = (int)(m.out & 3);
        const int head = min(total, (4 - h) & 3);
        const int bend = head + ((total - head) & ~3);
        if (act2) {
            uint32_t* ob = buf + h;
            if (diag >= head && diag + IT <= bend) {
#pragma unroll
                for (int q = 0; q < IT; ++q) {
                    ob[diag + q] = k[q];
                    if (V) ob[KW + diag + q] = vv[q];
                }
            } else {
#pragma unroll
                for (int q = 0; q < IT; ++q) {
                    const int e = diag + q;
                    if (e >= head && e < bend) {
                        ob[e] = k[q];
                        if (V) ob[KW + e] = vv[q];
                    } else if (e < total) {
                        dst_k[m.out + e] = k[q];
                        if (V) dst_v[m.out + e] = vv[q];
                    }
                }
            }
        }
        if (DC_M4_BARRIER_HANDOFF) {
            named_arrive<NC>(4 + b);                     // empty[b]
            continue;
        }
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(smem_addr(&empty[b]));
    }
}

}  // namespace dc
