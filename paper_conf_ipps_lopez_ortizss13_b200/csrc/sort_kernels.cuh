// sort_kernels.cuh -- sm_100a kernels of the breadth-first mergesort hot path.
//
// Alg 7 executed bottom-up, one data-parallel step per
// recursion level (Sec. 4.1-4.2):
//   NK1 blocksort  : base cases + the first log2(TILE) combine levels of every
//                    tile, entirely on chip (registers + shared memory);
//   NK2 partition  : merge-path co-rank of every output tile of one level
//                    (the "fn(id, param)" of Alg 3);
//   NK3 merge pass : one combine level over HBM, every CTA producing one
//                    aligned output tile of the merged pairs (Alg 7 lines 3-5).
// All merges are stable (left run wins ties, reading R5), so the
// result is the unique stable sorted permutation whatever the tile shape.
#pragma once
#include <cstdint>

namespace dc {

// ---------------------------------------------------------------- keys
// Keys travel as 32-bit patterns; only the comparison differs per type.
struct KeyU32 {
    static __device__ __forceinline__ bool lt(uint32_t a, uint32_t b) { return a < b; }
    static constexpr uint32_t kPad = 0xFFFFFFFFu;   // max key: pads sort last (stable)
};
struct KeyI32 {
    static __device__ __forceinline__ bool lt(uint32_t a, uint32_t b) {
        return (int32_t)a < (int32_t)b;
    }
    static constexpr uint32_t kPad = 0x7FFFFFFFu;
};
struct KeyF32 {
    static __device__ __forceinline__ bool lt(uint32_t a, uint32_t b) {
        return __uint_as_float(a) < __uint_as_float(b);
    }
    static constexpr uint32_t kPad = 0x7F800000u;   // +inf (NaN excluded by contract)
};

// Padded shared-memory index: one spare word per 32 makes the blocked
// (thread t owns [t*IT, t*IT+IT)) register<->smem transposes conflict-free.
__device__ __forceinline__ int pad32(int i) { return i + (i >> 5); }

// Words of a padded tile buffer; a multiple of 4 so that a second buffer
// placed right after it stays 16-byte aligned (uint4 accesses).
__host__ __device__ constexpr int padded_words(int tile) { return tile + tile / 32 + 4; }

// Merge-path co-rank (stable): the number i of elements of A among the first
// `diag` outputs of merge(A, B) where A wins ties:
//   largest i with  A[i-1] <= B[diag-i]  ... equivalently binary search with
//   "A[m] <= B[diag-1-m]  =>  lo = m+1".
template <class K, class LoadA, class LoadB>
__device__ __forceinline__ int merge_path(LoadA A, int a_len, LoadB B, int b_len, int diag) {
    int lo = max(0, diag - b_len);
    int hi = min(diag, a_len);
    while (lo < hi) {
        int m = (lo + hi) >> 1;
        if (!K::lt(B(diag - 1 - m), A(m))) lo = m + 1;
        else hi = m;
    }
    return lo;
}

template <class K>
__device__ __forceinline__ long long merge_path_global(const uint32_t* __restrict__ A,
                                                       long long a_len,
                                                       const uint32_t* __restrict__ B,
                                                       long long b_len, long long diag) {
    long long lo = diag - b_len > 0 ? diag - b_len : 0;
    long long hi = diag < a_len ? diag : a_len;
    while (lo < hi) {
        long long m = (lo + hi) >> 1;
        if (!K::lt(__ldg(B + (diag - 1 - m)), __ldg(A + m))) lo = m + 1;
        else hi = m;
    }
    return lo;
}

// ------------------------------------------------------------------ NK1
// One CTA sorts one tile of TILE = NT*IT keys (the last tile may be partial:
// it is padded with K::kPad, which sorts after every real key because every
// step is stable and the pads sit at the highest positions).
//   1. blocked load: thread t holds keys [t*IT, t*IT+IT) in registers;
//   2. leaves + levels with runs <= IT: stable odd-even transposition network
//      in registers;
//   3. levels with runs IT .. TILE/2: merge-path in padded shared memory, each
//      thread merging IT outputs serially;
//   4. transpose through shared memory, coalesced stores.
// With values (V): the network carries (key, tile-local index); the values
// are staged in shared memory and gathered by index at the end.
template <int NT, int IT, class K, bool V>
__global__ void __launch_bounds__(NT)
nk1_blocksort(const uint32_t* __restrict__ in_k, const uint32_t* __restrict__ in_v,
              uint32_t* __restrict__ out_k, uint32_t* __restrict__ out_v, long long n) {
    constexpr int TILE = NT * IT;
    constexpr int PADDED = padded_words(TILE);
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* sk = smem;                  // [PADDED] keys (padded index)
    uint32_t* si = smem + PADDED;         // [PADDED] indices (V only)
    uint32_t* sv = smem + 2 * PADDED;     // [TILE]   values (V only, linear)

    const int tid = threadIdx.x;
    const long long base = (long long)blockIdx.x * TILE;
    const int count = (int)min((long long)TILE, n - base);

    uint32_t k[IT];
    uint32_t ix[V ? IT : 1];

    // ---- 1. load (coalesced striped loads into padded smem, then blocked reads)
    if (count == TILE) {
        const uint4* src4 = reinterpret_cast<const uint4*>(in_k + base);
#pragma unroll
        for (int q = 0; q < IT / 4; ++q) {
            int e4 = q * NT + tid;            // uint4 index within tile
            uint4 v4 = __ldg(src4 + e4);
            int e = e4 * 4;
            sk[pad32(e + 0)] = v4.x;
            sk[pad32(e + 1)] = v4.y;
            sk[pad32(e + 2)] = v4.z;
            sk[pad32(e + 3)] = v4.w;
        }
        if (V) {
            const uint4* vsrc4 = reinterpret_cast<const uint4*>(in_v + base);
#pragma unroll
            for (int q = 0; q < IT / 4; ++q) {
                int e4 = q * NT + tid;
                reinterpret_cast<uint4*>(sv)[e4] = __ldg(vsrc4 + e4);
            }
        }
    } else {
#pragma unroll
        for (int q = 0; q < IT; ++q) {
            int e = q * NT + tid;
            sk[pad32(e)] = e < count ? __ldg(in_k + base + e) : K::kPad;
            if (V) sv[e] = e < count ? __ldg(in_v + base + e) : 0u;
        }
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < IT; ++j) {
        k[j] = sk[pad32(tid * IT + j)];
        if (V) ix[j] = tid * IT + j;
    }

    // ---- 2. in-register stable network (odd-even transposition sort)
#pragma unroll
    for (int r = 0; r < IT; ++r) {
#pragma unroll
        for (int j = r & 1; j + 1 < IT; j += 2) {
            bool sw = K::lt(k[j + 1], k[j]);
            uint32_t lo = sw ? k[j + 1] : k[j];
            uint32_t hi = sw ? k[j] : k[j + 1];
            k[j] = lo; k[j + 1] = hi;
            if (V) {
                uint32_t ilo = sw ? ix[j + 1] : ix[j];
                uint32_t ihi = sw ? ix[j] : ix[j + 1];
                ix[j] = ilo; ix[j + 1] = ihi;
            }
        }
    }

    // ---- 3. shared-memory merge levels: run width w -> 2w
#pragma unroll 1
    for (int w = IT; w < TILE; w *= 2) {
        __syncthreads();
#pragma unroll
        for (int j = 0; j < IT; ++j) {
            sk[pad32(tid * IT + j)] = k[j];
            if (V) si[pad32(tid * IT + j)] = ix[j];
        }
        __syncthreads();
        const int tpg = (2 * w) / IT;            // threads per merged pair
        const int s = (tid / tpg) * (2 * w);     // pair start
        const int diag = (tid % tpg) * IT;
        auto A = [&](int m) { return sk[pad32(s + m)]; };
        auto B = [&](int m) { return sk[pad32(s + w + m)]; };
        int i = merge_path<K>(A, w, B, w, diag);
        int ai = s + i, bi = s + w + diag - i;
        const int aend = s + w, bend = s + 2 * w;
        uint32_t a = sk[pad32(ai)];
        uint32_t b = sk[pad32(min(bi, TILE))];
#pragma unroll
        for (int j = 0; j < IT; ++j) {
            bool takeA = (bi >= bend) || ((ai < aend) && !K::lt(b, a));
            k[j] = takeA ? a : b;
            if (V) ix[j] = si[pad32(takeA ? ai : bi)];
            int nxt = takeA ? ++ai : ++bi;
            uint32_t v = sk[pad32(min(nxt, TILE))];
            if (takeA) a = v; else b = v;
        }
    }

    // ---- 4. store through smem: blocked write, striped coalesced read
    __syncthreads();
#pragma unroll
    for (int j = 0; j < IT; ++j) {
        sk[pad32(tid * IT + j)] = k[j];
        if (V) si[pad32(tid * IT + j)] = ix[j];
    }
    __syncthreads();
    if (count == TILE) {
        uint4* dst4 = reinterpret_cast<uint4*>(out_k + base);
#pragma unroll
        for (int q = 0; q < IT / 4; ++q) {
            int e4 = q * NT + tid, e = e4 * 4;
            dst4[e4] = make_uint4(sk[pad32(e)], sk[pad32(e + 1)], sk[pad32(e + 2)],
                                  sk[pad32(e + 3)]);
        }
        if (V) {
            uint4* vdst4 = reinterpret_cast<uint4*>(out_v + base);
#pragma unroll
            for (int q = 0; q < IT / 4; ++q) {
                int e4 = q * NT + tid, e = e4 * 4;
                vdst4[e4] = make_uint4(sv[si[pad32(e)]], sv[si[pad32(e + 1)]],
                                       sv[si[pad32(e + 2)]], sv[si[pad32(e + 3)]]);
            }
        }
    } else {
#pragma unroll
        for (int q = 0; q < IT; ++q) {
            int e = q * NT + tid;
            if (e < count) {
                out_k[base + e] = sk[pad32(e)];
                if (V) out_v[base + e] = sv[si[pad32(e)]];
            }
        }
    }
}

// ------------------------------------------------------------------ NK2
// Co-rank of the first output of every merge tile at run width w: tile j
// covers merged positions [j*TOUT, (j+1)*TOUT); its pair p starts at s = p*2w
// (TOUT divides 2w, so a tile never straddles two pairs).
template <class K>
__global__ void nk2_partition(const uint32_t* __restrict__ src, long long n, long long w,
                              int tout, int num_tiles, int* __restrict__ split) {
    int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= num_tiles) return;
    long long d0 = (long long)j * tout;
    long long s = (d0 / (2 * w)) * (2 * w);
    long long a_len = min(w, n - s);
    long long b_len = max(0LL, min(w, n - s - w));
    long long diag = d0 - s;
    split[j] = (int)merge_path_global<K>(src + s, a_len, src + s + a_len, b_len, diag);
}

// ------------------------------------------------------------------ NK3
// One output tile of TOUT = NT*IT merged keys per CTA.  The A and B pieces
// that feed the tile (known from the co-ranks) are staged in shared memory,
// each thread finds its own IT-output diagonal there and merges serially,
// results are transposed through shared memory for coalesced stores.
template <int NT, int IT, class K, bool V>
__global__ void __launch_bounds__(NT)
nk3_merge(const uint32_t* __restrict__ src_k, const uint32_t* __restrict__ src_v,
          uint32_t* __restrict__ dst_k, uint32_t* __restrict__ dst_v,
          const int* __restrict__ split, long long n, long long w) {
    constexpr int TOUT = NT * IT;
    constexpr int PADDED = padded_words(TOUT);
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* sk = smem;              // [PADDED]: inputs (linear) then outputs (padded)
    uint32_t* sv = smem + PADDED;     // [PADDED]: values, same layout (V only)

    const int tid = threadIdx.x;
    const int j = blockIdx.x;
    const long long d0 = (long long)j * TOUT;
    const long long s = (d0 / (2 * w)) * (2 * w);
    const long long a_len = min(w, n - s);
    const long long b_len = max(0LL, min(w, n - s - w));
    const long long dd0 = d0 - s;
    const long long dd1 = min(dd0 + TOUT, a_len + b_len);
    const int i0 = split[j];
    const int i1 = (dd1 == a_len + b_len) ? (int)a_len : split[j + 1];
    const int na = i1 - i0;
    const int nb = (int)(dd1 - dd0) - na;
    const uint32_t* gA = src_k + s + i0;
    const uint32_t* gB = src_k + s + a_len + (dd0 - i0);

    for (int q = tid; q < na; q += NT) sk[q] = __ldg(gA + q);
    for (int q = tid; q < nb; q += NT) sk[na + q] = __ldg(gB + q);
    if (V) {
        const uint32_t* vA = src_v + s + i0;
        const uint32_t* vB = src_v + s + a_len + (dd0 - i0);
        for (int q = tid; q < na; q += NT) sv[q] = __ldg(vA + q);
        for (int q = tid; q < nb; q += NT) sv[na + q] = __ldg(vB + q);
    }
    __syncthreads();

    const int total = na + nb;
    const int diag = min(tid * IT, total);
    auto A = [&](int m) { return sk[m]; };
    auto B = [&](int m) { return sk[na + m]; };
    int i = merge_path<K>(A, na, B, nb, diag);
    int ai = i, bi = na + diag - i;
    const int aend = na, bend = total;
    uint32_t k[IT];
    uint32_t vv[V ? IT : 1];
    uint32_t a = sk[min(ai, PADDED - 1)];
    uint32_t b = sk[min(bi, PADDED - 1)];
#pragma unroll
    for (int q = 0; q < IT; ++q) {
        bool takeA = (bi >= bend) || ((ai < aend) && !K::lt(b, a));
        k[q] = takeA ? a : b;
        if (V) vv[q] = sv[min(takeA ? ai : bi, PADDED - 1)];
        int nxt = takeA ? ++ai : ++bi;
        uint32_t v = sk[min(nxt, PADDED - 1)];
        if (takeA) a = v; else b = v;
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < IT; ++q) {
        sk[pad32(tid * IT + q)] = k[q];
        if (V) sv[pad32(tid * IT + q)] = vv[q];
    }
    __syncthreads();
    uint32_t* out = dst_k + d0;
    if (total == TOUT) {
        uint4* dst4 = reinterpret_cast<uint4*>(out);
#pragma unroll
        for (int q = 0; q < IT / 4; ++q) {
            int e4 = q * NT + tid, e = e4 * 4;
            dst4[e4] = make_uint4(sk[pad32(e)], sk[pad32(e + 1)], sk[pad32(e + 2)],
                                  sk[pad32(e + 3)]);
        }
        if (V) {
            uint4* vdst4 = reinterpret_cast<uint4*>(dst_v + d0);
#pragma unroll
            for (int q = 0; q < IT / 4; ++q) {
                int e4 = q * NT + tid, e = e4 * 4;
                vdst4[e4] = make_uint4(sv[pad32(e)], sv[pad32(e + 1)], sv[pad32(e + 2)],
                                       sv[pad32(e + 3)]);
            }
        }
    } else {
        for (int e = tid; e < total; e += NT) {
            out[e] = sk[pad32(e)];
            if (V) dst_v[d0 + e] = sv[pad32(e)];
        }
    }
}

}  // namespace dc
