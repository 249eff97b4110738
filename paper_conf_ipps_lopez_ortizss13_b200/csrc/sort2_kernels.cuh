// sort2_kernels.cuh -- two levels of the merge tree per HBM pass.
//
// A pass over runs of width w merges every group of four runs
// (R1 R2 R3 R4) into one run of 4w: M = merge(M1, M2), M1 = merge(R1, R2),
// M2 = merge(R3, R4), i.e. Alg 7's combine applied at two
// consecutive levels of the binary tree, with the intermediate runs M1, M2
// living only in shared memory.  The tree and every merge are the binary,
// stable ones of the one-level pass (earlier runs win ties), so the result is
// bit-identical; only the HBM traffic halves.
//   NK2a: co-ranks of every pair (R1,R2), (R3,R4) at multiples of a granule g
//         of its merged output (a table: M1[k*g] in O(1));
//   NK2b: for every output tile boundary d, the exact two-level co-rank
//         c = #M1 elements among the first d outputs -- coarse binary search on
//         the granule points, then a fine search inside one granule whose
//         element lookups are co-rank searches restricted to that granule --
//         plus the co-ranks x (R1 in M1 at c) and y (R3 in M2 at d - c);
//   NK3-2L: one output tile per CTA: the four pieces arrive by TMA, stage 1
//         merges them pairwise in shared memory (M1 and M2 pieces), stage 2
//         merges those, one TMA bulk store.
#pragma once
#include <cstdint>

namespace dc {

// A pair of sorted runs in global memory with a granule co-rank table:
// tab[k] = #A elements among the first min(k*g, la+lb) outputs of merge(A, B).
template <class K>
struct GPair {
    const uint32_t* A;
    long long la;
    const uint32_t* B;
    long long lb;
    const int* tab;
    long long g;

    // #A elements among the first p outputs (0 <= p <= la + lb)
    __device__ __forceinline__ long long corank(long long p) const {
        if (p <= 0) return 0;
        const long long m = la + lb;
        const long long k = p / g;
        const long long p0 = k * g;
        if (p == p0) return tab[k];
        const long long p1 = min(p0 + g, m);
        const long long i0 = tab[k], i1 = tab[k + 1];
        long long lo = max(max(i0, p - (p1 - i1)), max(0LL, p - lb));
        long long hi = min(min(i1, p - p0 + i0), min(p, la));
        while (lo < hi) {
            const long long mid = (lo + hi) >> 1;
            if (!K::lt(__ldg(B + (p - 1 - mid)), __ldg(A + mid))) lo = mid + 1;
            else hi = mid;
        }
        return lo;
    }
    // the output at position p (0 <= p < la + lb) given its co-rank i
    __device__ __forceinline__ uint32_t at_i(long long p, long long i) const {
        const long long j = p - i;
        if (i < la && (j >= lb || !K::lt(__ldg(B + j), __ldg(A + i)))) return __ldg(A + i);
        return __ldg(B + j);
    }
    __device__ __forceinline__ uint32_t at(long long p) const { return at_i(p, corank(p)); }
    // the last of the first q outputs (q >= 1) given the co-rank i at q:
    // the larger of A[i-1], B[q-i-1] (equal values are interchangeable here)
    __device__ __forceinline__ uint32_t last_i(long long q, long long i) const {
        const long long j = q - i;
        if (i == 0) return __ldg(B + j - 1);
        if (j == 0) return __ldg(A + i - 1);
        const uint32_t a = __ldg(A + i - 1), b = __ldg(B + j - 1);
        return K::lt(b, a) ? a : b;
    }
};

// Group geometry of a two-level pass over runs of width w.
__device__ __forceinline__ void group_runs(long long n, long long w, long long G, long long& s,
                                           long long& l1, long long& l2, long long& l3,
                                           long long& l4) {
    s = G * 4 * w;
    l1 = max(0LL, min(w, n - s));
    l2 = max(0LL, min(w, n - s - w));
    l3 = max(0LL, min(w, n - s - 2 * w));
    l4 = max(0LL, min(w, n - s - 3 * w));
}

// NK2a: granule table.  Thread (P, k): pair P = runs (2P, 2P+1) of width w,
// entry k = co-rank at min(k*g, m_P) (0 for pairs past the end).
template <class K>
__global__ void nk2a_granules(const uint32_t* __restrict__ src, long long n, long long w,
                              long long g, int K1, long long entries, int* __restrict__ tab) {
    const long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= entries) return;
    const long long P = e / K1, k = e % K1;
    const long long s = P * 2 * w;
    const long long la = max(0LL, min(w, n - s));
    const long long lb = max(0LL, min(w, n - s - w));
    const long long p = min(k * g, la + lb);
    tab[e] = (int)corank_global<K>(src + s, la, src + s + la, lb, p);
}

// NK2b: exact two-level co-ranks of every output tile boundary, one warp per
// boundary.  Tile j starts at global output j*T inside group G = j*T / 4w (T
// divides 4w, g divides T).  f(m) = M1[m] <= M2[d-1-m] is true then false on
// [lo, hi); c = its first false index: a coarse warp search over the granule
// points m = k*g (O(1) each from the table), then a fine warp search inside
// one granule (each probe two granule-restricted co-rank searches).  Writes
// bnd[3j..3j+2] = {c, x, y}: x = #R1 among the first c of M1, y = #R3 among
// the first d - c of M2.
template <class K>
__global__ void nk2b_partition2(const uint32_t* __restrict__ src, long long n, long long w,
                                long long T, long long g, int K1, const int* __restrict__ tab,
                                int num_tiles, int* __restrict__ bnd) {
    const int j = (int)(((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    if (j >= num_tiles) return;                       // warp-uniform
    const int lane = threadIdx.x & 31;
    const long long G = ((long long)j * T) / (4 * w);
    long long s, l1, l2, l3, l4;
    group_runs(n, w, G, s, l1, l2, l3, l4);
    const long long d = (long long)j * T - s;
    const GPair<K> M1{src + s, l1, src + s + l1, l2, tab + (2 * G) * K1, g};
    const GPair<K> M2{src + s + 2 * w, l3, src + s + 2 * w + l3, l4, tab + (2 * G + 1) * K1, g};
    const long long m1 = l1 + l2, m2 = l3 + l4;
    long long lo = max(0LL, d - m2), hi = min(d, m1);
    if (lo < hi) {
        const long long klo = (lo + g - 1) / g, khi = (hi - 1) / g;
        if (klo <= khi) {                             // coarse: granule points
            const long long a = warp_first_false(klo, khi + 1, [&](long long k) {
                const long long m = k * g;
                const uint32_t x1 = M1.at_i(m, M1.tab[k]);
                const long long q = d - m;            // multiple of g, >= 1
                const uint32_t y1 = M2.last_i(q, M2.tab[q / g]);
                return !K::lt(y1, x1);
            });
            if (a > klo) lo = max(lo, (a - 1) * g + 1);
            if (a <= khi) hi = min(hi, a * g);
        }
        lo = warp_first_false(lo, hi, [&](long long m) {   // fine: one granule
            const uint32_t x1 = M1.at(m);
            const uint32_t y1 = M2.at(d - 1 - m);
            return !K::lt(y1, x1);
        });
    }
    const long long c = lo;
    if (lane == 0) bnd[3 * j + 0] = (int)c;
    if (lane == 1) bnd[3 * j + 1] = (int)M1.corank(c);
    if (lane == 2) bnd[3 * j + 2] = (int)M2.corank(d - c);
}

// NK3-2L: tile J of the two-level pass (keys only), T = NT*IT outputs.
// NT + 32 threads: stage 1 has up to NT + 1 windows of IT outputs (the M1
// and M2 pieces are windowed separately).  Stage-1 results wait in registers
// and then overwrite the staging buffer, so one T-sized buffer serves the
// four pieces, the two intermediate pieces and the output tile.
template <int NT, int IT, class K>
__global__ void __launch_bounds__(NT + 32)
nk3_merge2(const uint32_t* __restrict__ src, uint32_t* __restrict__ dst, long long n, long long w,
           const int* __restrict__ bnd) {
    constexpr int T = NT * IT;
    extern __shared__ __align__(16) uint32_t st[];   // nk3_2l_words(T, IT) words
    __shared__ __align__(8) uint64_t bar;
    const uint32_t ST = smem_addr(st), BAR = smem_addr(&bar);
    const int tid = threadIdx.x;
    const long long J = blockIdx.x;
    const long long G = (J * T) / (4 * w);
    long long s, l1, l2, l3, l4;
    group_runs(n, w, G, s, l1, l2, l3, l4);
    const long long m1 = l1 + l2, m2 = l3 + l4;
    const long long d0 = J * T - s;
    const long long d1 = min(d0 + T, m1 + m2);
    const long long c0 = bnd[3 * J], x0 = bnd[3 * J + 1], y0 = bnd[3 * J + 2];
    long long c1, x1, y1;
    if (d1 == m1 + m2) { c1 = m1; x1 = l1; y1 = l3; }
    else { c1 = bnd[3 * J + 3]; x1 = bnd[3 * J + 4]; y1 = bnd[3 * J + 5]; }
    // the four pieces (global element ranges)
    const long long g0[4] = {s + x0, s + l1 + (c0 - x0), s + 2 * w + y0,
                             s + 2 * w + l3 + ((d0 - c0) - y0)};
    const int len[4] = {(int)(x1 - x0), (int)((c1 - x1) - (c0 - x0)), (int)(y1 - y0),
                        (int)(((d1 - c1) - y1) - ((d0 - c0) - y0))};
    int off[4];                            // word offset of each piece's aligned superset
    {
        int o = 0;
        for (int p = 0; p < 4; ++p) {
            off[p] = o;
            o = (o + (int)(g0[p] & 3) + len[p] + 1 + 3) & ~3;
        }
    }
    const long long n4 = n & ~3LL;
    if (tid == 0) {
        mbar_init(BAR, 1);
        uint32_t bytes = 0;
        for (int p = 0; p < 4; ++p) bytes += piece_bytes(g0[p], g0[p] + len[p], n4);
        mbar_arrive_expect_tx(BAR, bytes);
        for (int p = 0; p < 4; ++p) stage_piece(src, g0[p], g0[p] + len[p], n4, off[p], ST, BAR);
    }
    for (int p = 0; p < 4; ++p) {          // elements at or past n4 (array tail only)
        if (g0[p] + len[p] > n4) {
            for (long long e = max(g0[p], n4) + tid; e < g0[p] + len[p]; e += NT + 32)
                st[off[p] + (int)(g0[p] & 3) + (e - g0[p])] = src[e];
        }
    }
    __syncthreads();
    mbar_wait(BAR, 0);

    // stage 1 (registers): window tid of [M1 piece windows | M2 piece windows]
    const int n1 = len[0] + len[1], n2 = len[2] + len[3];
    const int w1 = (n1 + IT - 1) / IT, w2 = (n2 + IT - 1) / IT;
    uint32_t k[IT], srcb[IT];
    int out0 = 0, valid = 0;
    const int o2 = n1 + 4;                 // intermediate layout: M1 piece | 4 slack | M2 piece
    if (tid < w1 + w2) {
        const bool first = tid < w1;
        const int pa = first ? 0 : 2;
        const uint32_t A = ST + 4u * (off[pa] + (int)(g0[pa] & 3));
        const uint32_t B = ST + 4u * (off[pa + 1] + (int)(g0[pa + 1] & 3));
        const int na = len[pa], nb = len[pa + 1];
        const int diag = (first ? tid : tid - w1) * IT;
        const int i = corank_smem<K>(A, na, B, nb, diag);
        serial_merge<K, IT, false>(A + 4u * i, A + 4u * na, B + 4u * (diag - i), B + 4u * nb, k,
                                   srcb);
        valid = min(IT, na + nb - diag);
        out0 = (first ? 0 : o2) + diag;
    }
    __syncthreads();                       // all pieces consumed
#pragma unroll
    for (int q = 0; q < IT; ++q)
        if (q < valid) st[out0 + q] = k[q];
    __syncthreads();

    // stage 2: merge the M1 and M2 pieces -> T outputs, blocked into `st`
    const int total = n1 + n2;
    const int diag = tid * IT;
    if (tid < NT && diag < total) {
        const int i = corank_smem<K>(ST, n1, ST + 4u * o2, n2, diag);
        serial_merge<K, IT, false>(ST + 4u * i, ST + 4u * n1, ST + 4u * (o2 + diag - i),
                                   ST + 4u * (o2 + n2), k, srcb);
    }
    __syncthreads();
    if (tid < NT && diag < total) {
#pragma unroll
        for (int q = 0; q < IT; ++q) st[diag + q] = k[q];
    }
    fence_proxy_async_smem();
    __syncthreads();
    store_tile(dst + J * T, st, 0, total);
}

// Shared words of nk3_merge2: the four staged pieces (T + 28 with alignment
// slack), the intermediate pieces (T + 4) and the serial merges' past-the-end
// reads (up to IT words), rounded to 16 bytes.
__host__ __device__ constexpr int nk3_2l_words(int T, int IT) { return (T + IT + 64 + 3) / 4 * 4; }

}  // namespace dc
