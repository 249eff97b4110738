// mg_kernels.cuh -- the top log2(G) levels of a G-way sharded sort.
//
// Not in the paper (its experiments use one GPU; it notes the
// method "could easily be extended to multiple gpu cards").
// Rank r holds the shard of global positions [r*m, (r+1)*m) and has sorted it
// (levels >= log2 G are independent subproblems).  The top log2 G levels
// become one exchange step:
//   a7  exact splitters: every S-th key of every sorted shard is a candidate;
//       candidates are ordered by the composite key (key, rank, position),
//       which is exactly the order of the global stable sort.  Each rank
//       counts its elements below every candidate (mg_count), the counts are
//       summed across ranks (all-reduce) into global ranks, every boundary
//       k_d = d*m is bracketed by two consecutive candidates (mg_brackets),
//       the < S elements of each rank between them are exchanged
//       (mg_windows + all-gather) and the exact split of every boundary
//       follows (mg_split_matrix): c[r][d] = number of rank-r elements among
//       the first k_d of the global order;
//   a8  all-to-all of the ranges [c[r][d], c[r][d+1]) (torch.distributed /
//       NCCL over NVLink);
//   a9  local stable G-way merge of the received runs (earlier rank wins
//       ties) with the merge-path kernels of sort_kernels.cuh.
#pragma once
#include <cstdint>

#include "sort_kernels.cuh"   // warp_first_false

namespace dc {

// a7 (1/4): every stride-th key of a sorted shard.
__global__ void mg_sample(const uint32_t* __restrict__ keys, long long stride, long long count,
                          uint32_t* __restrict__ out) {
    const long long j = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < count) out[j] = keys[j * stride];
}

template <class K>
__device__ __forceinline__ long long lower_bound_g(const uint32_t* __restrict__ a, long long n,
                                                   uint32_t v) {
    long long lo = 0, hi = n;   // first i with !(a[i] < v)
    while (lo < hi) {
        const long long mid = (lo + hi) >> 1;
        if (K::lt(__ldg(a + mid), v)) lo = mid + 1; else hi = mid;
    }
    return lo;
}
template <class K>
__device__ __forceinline__ long long upper_bound_g(const uint32_t* __restrict__ a, long long n,
                                                   uint32_t v) {
    long long lo = 0, hi = n;   // first i with v < a[i]
    while (lo < hi) {
        const long long mid = (lo + hi) >> 1;
        if (!K::lt(v, __ldg(a + mid))) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// a7 (2/4): composite count.  Candidate c (rank-major: c = owner*q + j) is
// the element (cand[c], owner, j*stride).  Elements of this rank (`me`)
// strictly below it in (key, rank, position) order:
//   me <  owner: keys <= key;   me == owner: the j*stride elements before it;
//   me >  owner: keys <  key.
template <class K>
__global__ void mg_count(const uint32_t* __restrict__ keys, long long n, int me,
                         const uint32_t* __restrict__ cand, long long q, long long stride,
                         long long cands, int64_t* __restrict__ out) {
    const long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= cands) return;
    const int owner = (int)(c / q);
    const uint32_t v = cand[c];
    long long r;
    if (me < owner) r = upper_bound_g<K>(keys, n, v);
    else if (me == owner) r = (c % q) * stride;
    else r = lower_bound_g<K>(keys, n, v);
    out[c] = r;
}

// a7 (3/4a): bracket every boundary k_d = d*m (d = 1..G-1) by the candidates
// of largest global rank < k_d (lo) and smallest global rank >= k_d (hi).
// Global ranks are distinct (candidates are distinct elements); packed as
// ((rank + 1) << 24) | c so one 64-bit atomic max / min finds both.
// Every candidate's packed value is reduced within its warp first (max of
// the ones below k_d, min of the others), so one lane per warp issues the
// atomics: the G-1 addresses see cands/32 atomics each instead of cands
// (ncu, loopback G = 4, 2^25 keys: 12-20 us of contended atomics before).
__global__ void mg_brackets(const int64_t* __restrict__ R, long long cands, int G, long long m,
                            unsigned long long* __restrict__ lo_pack,
                            unsigned long long* __restrict__ hi_pack) {
    const long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const bool valid = c < cands;                      // every lane takes part in the shuffles
    const long long rc = valid ? R[c] : 0;
    const unsigned long long packed = ((unsigned long long)(rc + 1) << 24) | (unsigned long long)c;
    for (int d = 1; d < G; ++d) {
        const long long k = (long long)d * m;
        unsigned long long lo = (valid && rc < k) ? packed : 0ULL;
        unsigned long long hi = (valid && rc >= k) ? packed : ~0ULL;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            lo = max(lo, __shfl_xor_sync(0xffffffffu, lo, o));
            hi = min(hi, __shfl_xor_sync(0xffffffffu, hi, o));
        }
        if ((threadIdx.x & 31) == 0) {
            if (lo != 0ULL) atomicMax(lo_pack + d, lo);
            if (hi != ~0ULL) atomicMin(hi_pack + d, hi);
        }
    }
}

// Send-buffer layout of one rank (uint32 words): for d = 1..G-1 a header of
// three int64 {lo, len, t} at words [6(d-1), 6d), then the window keys of
// boundary d at words hdr + (d-1)*wcap, hdr = 6(G-1).  The total is rounded
// up to a multiple of 4 words, so every rank's buffer in the all-gathered
// array starts 16-byte aligned and its int64 headers are aligned loads for
// any stride (an odd stride with G even used to misalign every odd rank).
__host__ __device__ constexpr long long mg_sendbuf_words(int G, long long wcap) {
    return (6LL * (G - 1) + (long long)(G - 1) * wcap + 3) / 4 * 4;
}

// a7 (3/4b): one CTA per boundary d.  This rank's elements strictly between
// the two bracketing candidates form positions [lo, hi) of its shard
// (hi - lo < stride); t = number of window elements (over all ranks) that
// belong to the first k_d.  Writes header + keys into the send buffer.
__global__ void mg_windows(const uint32_t* __restrict__ keys, long long n, int me, int G,
                           long long m, const int64_t* __restrict__ C,
                           const int64_t* __restrict__ R, long long q, long long wcap,
                           const unsigned long long* __restrict__ lo_pack,
                           const unsigned long long* __restrict__ hi_pack,
                           uint32_t* __restrict__ sendbuf, int* __restrict__ err) {
    const int d = blockIdx.x + 1;
    const unsigned long long lp = lo_pack[d], hp = hi_pack[d];
    const bool has_lo = lp != 0ULL, has_hi = hp != ~0ULL;
    const long long a = (long long)(lp & 0xFFFFFFULL), b = (long long)(hp & 0xFFFFFFULL);
    const long long lo = has_lo ? C[a] + ((int)(a / q) == me ? 1 : 0) : 0;
    const long long hi = has_hi ? C[b] : n;
    const long long t = (long long)d * m - (has_lo ? R[a] + 1 : 0);
    long long len = hi - lo;
    if (len < 0 || len > wcap) {            // cannot happen for sorted shards
        if (threadIdx.x == 0) atomicExch(err, 1);
        len = 0;
    }
    long long* hdr = reinterpret_cast<long long*>(sendbuf);
    if (threadIdx.x == 0) {
        hdr[3 * (d - 1) + 0] = lo;
        hdr[3 * (d - 1) + 1] = len;
        hdr[3 * (d - 1) + 2] = t;
    }
    uint32_t* w = sendbuf + 6LL * (G - 1) + (long long)(d - 1) * wcap;
    for (long long e = threadIdx.x; e < len; e += blockDim.x) w[e] = keys[lo + e];
}

// Position of window element (r, p) in the stable merge of the G windows of
// one boundary (key, then rank): p + sum_{r'<r} #{<= key} + sum_{r'>r} #{< key}.
template <class K>
__device__ __forceinline__ long long merged_rank(const uint32_t* s, const int* off,
                                                 const long long* len, int G, int r, long long p) {
    const uint32_t v = s[off[r] + p];
    long long acc = p;
    for (int r2 = 0; r2 < G; ++r2) {
        if (r2 == r) continue;
        const uint32_t* a = s + off[r2];
        long long lo = 0, hi = len[r2];
        if (r2 < r) {          // upper bound: earlier ranks win ties
            while (lo < hi) {
                const long long mid = (lo + hi) >> 1;
                if (!K::lt(v, a[mid])) lo = mid + 1; else hi = mid;
            }
        } else {               // lower bound
            while (lo < hi) {
                const long long mid = (lo + hi) >> 1;
                if (K::lt(a[mid], v)) lo = mid + 1; else hi = mid;
            }
        }
        acc += lo;
    }
    return acc;
}

// a7 (4/4): one CTA per boundary d.  `gathered` holds the G send buffers
// back to back (rank order).  The G windows are staged in shared memory;
// thread r < G finds cnt_r = #(rank-r window elements among the first t of
// the merged windows) by binary search on its window position.  Writes
// cmat[r][d] = lo_r + cnt_r; cmat[r][0] = 0 and cmat[r][G] = m (G x (G+1)).
template <class K>
__global__ void mg_split_matrix(const uint32_t* __restrict__ gathered, int G, long long m,
                                long long wcap, int64_t* __restrict__ cmat) {
    extern __shared__ uint32_t win[];   // G * wcap words
    __shared__ int off[64];
    __shared__ long long len[64], lo[64];
    const int d = blockIdx.x + 1;
    const long long words = mg_sendbuf_words(G, wcap);
    if (threadIdx.x < G) {
        const int r = threadIdx.x;
        const long long* hdr = reinterpret_cast<const long long*>(gathered + r * words);
        lo[r] = hdr[3 * (d - 1) + 0];
        len[r] = hdr[3 * (d - 1) + 1];
        off[r] = (int)(r * wcap);
    }
    __syncthreads();
    for (int r = 0; r < G; ++r) {
        const uint32_t* w = gathered + r * words + 6LL * (G - 1) + (long long)(d - 1) * wcap;
        for (long long e = threadIdx.x; e < len[r]; e += blockDim.x) win[off[r] + e] = w[e];
    }
    __syncthreads();
    const long long t = reinterpret_cast<const long long*>(gathered)[3 * (d - 1) + 2];
    // one warp per rank r: cnt = first p with merged_rank(r, p) >= t, found by
    // a 33-ary warp search (32 probes per round, ~3 rounds for a window of
    // 4096) instead of one thread's binary search (12 dependent probes, each
    // G-1 inner searches); ncu, loopback G = 4: ~110 us per launch before.
    const int lane = threadIdx.x & 31;
    for (int r = threadIdx.x >> 5; r < G; r += blockDim.x >> 5) {
        const long long cnt = warp_first_false(0, len[r], [&](long long p) {
            return merged_rank<K>(win, off, len, G, r, p) < t;
        });
        if (lane == 0) {
            cmat[r * (G + 1) + d] = lo[r] + cnt;
            if (d == 1) {
                cmat[r * (G + 1) + 0] = 0;
                cmat[r * (G + 1) + G] = m;
            }
        }
    }
}

}  // namespace dc
