// sort_kernels.cuh -- sm_100a kernels of the breadth-first mergesort hot path.
//
// Alg 7 executed bottom-up, one data-parallel step per
// recursion level (Sec. 4.1-4.2):
//   NK1 blocksort  : base cases + the first combine levels of every tile,
//                    entirely on chip (registers + shared memory);
//   NK2 partition  : merge-path co-rank of every output tile of one level
//                    (the "fn(id, param)" of Alg 3);
//   NK3 merge pass : one combine level over HBM, every CTA producing one
//                    aligned output tile of the merged pairs (Alg 7 lines 3-5).
// All merges are stable (left run wins ties, reading R5), so the
// result is the unique stable sorted permutation whatever the tile shape.
//
// Items per thread (IT) are odd: a thread's IT consecutive elements then sit
// at stride IT words, which hits 32 distinct banks, so the blocked
// register<->shared transposes are conflict-free with a plain linear layout
// and the serial merge walks shared memory with +4-byte address steps.
#pragma once
#include <cstdint>

namespace dc {

// ---------------------------------------------------------------- keys
// Keys travel as 32-bit patterns; only the comparison differs per type.
struct KeyU32 {
    static __device__ __forceinline__ bool lt(uint32_t a, uint32_t b) { return a < b; }
    static __device__ __forceinline__ uint32_t mn(uint32_t a, uint32_t b) { return min(a, b); }
    static __device__ __forceinline__ uint32_t mx(uint32_t a, uint32_t b) { return max(a, b); }
    static constexpr uint32_t kPad = 0xFFFFFFFFu;   // max key: pads sort last (stable)
    static constexpr bool kNeedStable = false;       // equal keys are identical bits
};
struct KeyI32 {
    static __device__ __forceinline__ bool lt(uint32_t a, uint32_t b) {
        return (int32_t)a < (int32_t)b;
    }
    static __device__ __forceinline__ uint32_t mn(uint32_t a, uint32_t b) {
        return (uint32_t)min((int32_t)a, (int32_t)b);
    }
    static __device__ __forceinline__ uint32_t mx(uint32_t a, uint32_t b) {
        return (uint32_t)max((int32_t)a, (int32_t)b);
    }
    static constexpr uint32_t kPad = 0x7FFFFFFFu;
    static constexpr bool kNeedStable = false;
};
struct KeyF32 {
    static __device__ __forceinline__ bool lt(uint32_t a, uint32_t b) {
        return __uint_as_float(a) < __uint_as_float(b);
    }
    static __device__ __forceinline__ uint32_t mn(uint32_t a, uint32_t b) { return lt(b, a) ? b : a; }
    static __device__ __forceinline__ uint32_t mx(uint32_t a, uint32_t b) { return lt(b, a) ? a : b; }
    static constexpr uint32_t kPad = 0x7F800000u;   // +inf (NaN excluded by contract)
    static constexpr bool kNeedStable = true;        // +0.0 / -0.0 are equal, distinct bits
};

// ------------------------------------------------------- shared memory
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ uint32_t lds(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
}

// Words of a tile buffer: the tile plus `slack` words for the past-the-end
// reads of the serial merge, rounded to 16 bytes so a following buffer stays
// aligned.
__host__ __device__ constexpr int tile_words(int tile, int slack) {
    return (tile + slack + 1 + 3) / 4 * 4;
}

// ---------------------------------------------------- merge primitives

// Merge-path co-rank (stable): number of A elements among the first `diag`
// outputs of merge(A, B) where A wins ties.  Binary search with the rule
// "A[m] <= B[diag-1-m]  =>  lo = m+1".  A and B given as shared byte addresses.
template <class K>
__device__ __forceinline__ int corank_smem(uint32_t A, int a_len, uint32_t B, int b_len, int diag) {
    int lo = max(0, diag - b_len);
    int hi = min(diag, a_len);
    while (lo < hi) {
        int m = (lo + hi) >> 1;
        uint32_t am = lds(A + 4u * m);
        uint32_t bm = lds(B + 4u * (diag - 1 - m));
        if (!K::lt(bm, am)) lo = m + 1;
        else hi = m;
    }
    return lo;
}

template <class K>
__device__ __forceinline__ long long corank_global(const uint32_t* __restrict__ A, long long a_len,
                                                   const uint32_t* __restrict__ B, long long b_len,
                                                   long long diag) {
    long long lo = diag - b_len > 0 ? diag - b_len : 0;
    long long hi = diag < a_len ? diag : a_len;
    while (lo < hi) {
        long long m = (lo + hi) >> 1;
        if (!K::lt(__ldg(B + (diag - 1 - m)), __ldg(A + m))) lo = m + 1;
        else hi = m;
    }
    return lo;
}

// Serial stable merge of IT outputs from shared memory.  ai/bi: byte addresses
// of the current A and B heads; a_end/b_end: byte addresses one past the runs.
// Reads at a_end / b_end are allowed (slack) and never selected.  With SRC the
// byte address each output came from is recorded (to gather values later).
template <class K, int IT, bool SRC>
__device__ __forceinline__ void serial_merge(uint32_t ai, uint32_t a_end, uint32_t bi,
                                             uint32_t b_end, uint32_t (&out)[IT],
                                             uint32_t (&src)[IT]) {
    uint32_t a = lds(ai), b = lds(bi);
    const uint32_t c0 = ai + bi;   // ai + bi grows by exactly 4 bytes per output
#pragma unroll
    for (int j = 0; j < IT; ++j) {
        const bool p = (ai >= a_end) | ((bi < b_end) & K::lt(b, a));   // take B
        out[j] = p ? b : a;
        if (SRC) src[j] = p ? bi : ai;
        if (!p) ai += 4u;
        bi = c0 + 4u * (j + 1) - ai;
        const uint32_t v = lds(p ? bi : ai);
        if (p) b = v; else a = v;
    }
}

// ------------------------------------------------- in-register networks

// Batcher odd-even merge sort network on N elements (implicitly padded with
// +inf to a power of two; comparators touching the padding are dropped).
template <int N, class CAS>
__device__ __forceinline__ void batcher_network(CAS&& cas) {
    constexpr int P2 = (N <= 1) ? 1 : (N <= 2) ? 2 : (N <= 4) ? 4 : (N <= 8) ? 8
                     : (N <= 16) ? 16 : (N <= 32) ? 32 : 64;
#pragma unroll
    for (int p = 1; p < P2; p <<= 1)
#pragma unroll
        for (int k = p; k >= 1; k >>= 1)
#pragma unroll
            for (int j = k % p; j + k < P2; j += 2 * k)
#pragma unroll
                for (int i = 0; i < k; ++i)
                    if (i + j + k < N && (i + j) / (2 * p) == (i + j + k) / (2 * p))
                        cas(i + j, i + j + k);
}

// Sort IT keys held by one thread.  Keys-only u32/i32 (stability unobservable)
// use Batcher's network with min/max; otherwise a stable odd-even
// transposition network carrying the indices.
template <class K, int IT, bool V>
__device__ __forceinline__ void thread_sort(uint32_t (&k)[IT], uint32_t (&ix)[IT]) {
    if constexpr (!V && !K::kNeedStable) {
        batcher_network<IT>([&](int x, int y) {
            const uint32_t lo = K::mn(k[x], k[y]);
            const uint32_t hi = K::mx(k[x], k[y]);
            k[x] = lo;
            k[y] = hi;
        });
    } else {
#pragma unroll
        for (int r = 0; r < IT; ++r) {
#pragma unroll
            for (int j = r & 1; j + 1 < IT; j += 2) {
                const bool sw = K::lt(k[j + 1], k[j]);
                const uint32_t lo = sw ? k[j + 1] : k[j];
                const uint32_t hi = sw ? k[j] : k[j + 1];
                k[j] = lo;
                k[j + 1] = hi;
                if (V) {
                    const uint32_t ilo = sw ? ix[j + 1] : ix[j];
                    const uint32_t ihi = sw ? ix[j] : ix[j + 1];
                    ix[j] = ilo;
                    ix[j + 1] = ihi;
                }
            }
        }
    }
}

// ------------------------------------------------------------------ NK1
// One CTA sorts one tile of TILE = NT*IT keys (the last tile may be partial:
// it is padded with K::kPad, which sorts after every real key because every
// step is stable and the pads sit at the highest positions).
//   1. coalesced 128-bit loads into shared memory, blocked reads (thread t
//      holds keys [t*IT, t*IT+IT));
//   2. leaves + the levels inside a thread: in-register network;
//   3. levels with runs IT .. TILE/2: merge-path in shared memory, each
//      thread merging IT outputs serially;
//   4. transpose through shared memory, coalesced 128-bit stores.
// With values (V): the merges carry the tile-local index of every key; the
// values wait in shared memory and are gathered by index at the end.
template <int NT, int IT, class K, bool V>
__global__ void __launch_bounds__(NT)
nk1_blocksort(const uint32_t* __restrict__ in_k, const uint32_t* __restrict__ in_v,
              uint32_t* __restrict__ out_k, uint32_t* __restrict__ out_v, long long n) {
    static_assert(IT % 2 == 1, "odd items per thread keep the blocked layout conflict-free");
    constexpr int TILE = NT * IT;
    static_assert(TILE % 4 == 0, "tile must be a whole number of uint4");
    constexpr int TW = tile_words(TILE, 0);
    constexpr int Q4 = (TILE / 4 + NT - 1) / NT;     // uint4 per thread (striped)
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* sk = smem;              // [TW] keys
    uint32_t* si = smem + TW;         // [TW] tile-local indices (V only)
    uint32_t* sv = smem + 2 * TW;     // [TW] values, by original position (V only)
    const uint32_t SK = smem_addr(sk);
    constexpr uint32_t SI_OFF = TW * 4;

    const int tid = threadIdx.x;
    const long long base = (long long)blockIdx.x * TILE;
    const int count = (int)min((long long)TILE, n - base);

    // ---- 1. load
    if (count == TILE) {
        const uint4* src4 = reinterpret_cast<const uint4*>(in_k + base);
#pragma unroll
        for (int q = 0; q < Q4; ++q) {
            const int e4 = q * NT + tid;
            if (e4 < TILE / 4) reinterpret_cast<uint4*>(sk)[e4] = __ldg(src4 + e4);
        }
        if (V) {
            const uint4* vsrc4 = reinterpret_cast<const uint4*>(in_v + base);
#pragma unroll
            for (int q = 0; q < Q4; ++q) {
                const int e4 = q * NT + tid;
                if (e4 < TILE / 4) reinterpret_cast<uint4*>(sv)[e4] = __ldg(vsrc4 + e4);
            }
        }
    } else {
#pragma unroll 4
        for (int e = tid; e < TILE; e += NT) {
            sk[e] = e < count ? __ldg(in_k + base + e) : K::kPad;
            if (V) sv[e] = e < count ? __ldg(in_v + base + e) : 0u;
        }
    }
    __syncthreads();
    uint32_t k[IT];
    uint32_t ix[IT];
#pragma unroll
    for (int j = 0; j < IT; ++j) {
        k[j] = sk[tid * IT + j];
        ix[j] = tid * IT + j;
    }

    // ---- 2. leaves + in-thread levels
    thread_sort<K, IT, V>(k, ix);

    // ---- 3. shared-memory merge levels: run width w -> 2w
#pragma unroll 1
    for (int w = IT; w < TILE; w *= 2) {
        __syncthreads();
#pragma unroll
        for (int j = 0; j < IT; ++j) {
            sk[tid * IT + j] = k[j];
            if (V) si[tid * IT + j] = ix[j];
        }
        __syncthreads();
        const int tpg = (2 * w) / IT;            // threads per merged pair
        const int s = (tid / tpg) * (2 * w);     // pair start
        const int diag = (tid % tpg) * IT;
        const uint32_t A = SK + 4u * s, B = A + 4u * w;
        const int i = corank_smem<K>(A, w, B, w, diag);
        uint32_t src[IT];
        serial_merge<K, IT, V>(A + 4u * i, B, B + 4u * (diag - i), B + 4u * w, k, src);
        if (V) {
#pragma unroll
            for (int j = 0; j < IT; ++j) ix[j] = lds(src[j] + SI_OFF);
        }
    }

    // ---- 4. store through shared memory: blocked write, striped 128-bit reads
    __syncthreads();
#pragma unroll
    for (int j = 0; j < IT; ++j) {
        sk[tid * IT + j] = k[j];
        if (V) si[tid * IT + j] = ix[j];
    }
    __syncthreads();
    if (count == TILE) {
        uint4* dst4 = reinterpret_cast<uint4*>(out_k + base);
#pragma unroll
        for (int q = 0; q < Q4; ++q) {
            const int e4 = q * NT + tid;
            if (e4 < TILE / 4) dst4[e4] = reinterpret_cast<const uint4*>(sk)[e4];
        }
        if (V) {
            uint4* vdst4 = reinterpret_cast<uint4*>(out_v + base);
#pragma unroll
            for (int q = 0; q < Q4; ++q) {
                const int e4 = q * NT + tid;
                if (e4 < TILE / 4) {
                    const uint4 s4 = reinterpret_cast<const uint4*>(si)[e4];
                    vdst4[e4] = make_uint4(sv[s4.x], sv[s4.y], sv[s4.z], sv[s4.w]);
                }
            }
        }
    } else {
        for (int e = tid; e < count; e += NT) {
            out_k[base + e] = sk[e];
            if (V) out_v[base + e] = sv[si[e]];
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
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= num_tiles) return;
    const long long d0 = (long long)j * tout;
    const long long s = (d0 / (2 * w)) * (2 * w);
    const long long a_len = min(w, n - s);
    const long long b_len = max(0LL, min(w, n - s - w));
    split[j] = (int)corank_global<K>(src + s, a_len, src + s + a_len, b_len, d0 - s);
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
    static_assert(IT % 2 == 1, "odd items per thread keep the blocked layout conflict-free");
    constexpr int TOUT = NT * IT;
    static_assert(TOUT % 4 == 0, "tile must be a whole number of uint4");
    constexpr int TW = tile_words(TOUT, IT);
    constexpr int Q = (TOUT + NT - 1) / NT;
    constexpr int Q4 = (TOUT / 4 + NT - 1) / NT;
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* sk = smem;          // [TW]: A piece | B piece, then the merged tile
    uint32_t* sv = smem + TW;     // [TW]: values, same layout (V only)
    const uint32_t SK = smem_addr(sk);
    constexpr uint32_t SV_OFF = TW * 4;

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
    const int total = (int)(dd1 - dd0);
    const uint32_t* gA = src_k + s + i0;
    const uint32_t* gB = src_k + s + a_len + (dd0 - i0) - na;   // indexed by e in [na, total)

#pragma unroll
    for (int q = 0; q < Q; ++q) {
        const int e = q * NT + tid;
        if (e < total) sk[e] = __ldg(e < na ? gA + e : gB + e);
    }
    if (V) {
        const uint32_t* vA = src_v + s + i0;
        const uint32_t* vB = src_v + s + a_len + (dd0 - i0) - na;
#pragma unroll
        for (int q = 0; q < Q; ++q) {
            const int e = q * NT + tid;
            if (e < total) sv[e] = __ldg(e < na ? vA + e : vB + e);
        }
    }
    __syncthreads();

    const int diag = min(tid * IT, total);
    const int i = corank_smem<K>(SK, na, SK + 4u * na, total - na, diag);
    uint32_t k[IT], src[IT];
    serial_merge<K, IT, V>(SK + 4u * i, SK + 4u * na, SK + 4u * (na + diag - i),
                           SK + 4u * total, k, src);
    uint32_t vv[IT];
    if (V) {
#pragma unroll
        for (int q = 0; q < IT; ++q) vv[q] = lds(src[q] + SV_OFF);
    }
    __syncthreads();
#pragma unroll
    for (int q = 0; q < IT; ++q) {
        sk[tid * IT + q] = k[q];
        if (V) sv[tid * IT + q] = vv[q];
    }
    __syncthreads();
    if (total == TOUT) {
        uint4* dst4 = reinterpret_cast<uint4*>(dst_k + d0);
#pragma unroll
        for (int q = 0; q < Q4; ++q) {
            const int e4 = q * NT + tid;
            if (e4 < TOUT / 4) dst4[e4] = reinterpret_cast<const uint4*>(sk)[e4];
        }
        if (V) {
            uint4* vdst4 = reinterpret_cast<uint4*>(dst_v + d0);
#pragma unroll
            for (int q = 0; q < Q4; ++q) {
                const int e4 = q * NT + tid;
                if (e4 < TOUT / 4) vdst4[e4] = reinterpret_cast<const uint4*>(sv)[e4];
            }
        }
    } else {
        for (int e = tid; e < total; e += NT) {
            dst_k[d0 + e] = sk[e];
            if (V) dst_v[d0 + e] = sv[e];
        }
    }
}

}  // namespace dc
