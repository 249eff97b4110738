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
#include <type_traits>
#include <utility>

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
// The comparator list is generated at compile time and expanded by a fold
// expression, so every register index is a constant (the arrays stay in
// registers; a runtime-unrolled loop nest of this size spills to local memory).
template <int N>
struct BatcherPairs {
    static constexpr int P2 = (N <= 1) ? 1 : (N <= 2) ? 2 : (N <= 4) ? 4 : (N <= 8) ? 8
                            : (N <= 16) ? 16 : (N <= 32) ? 32 : (N <= 64) ? 64 : 128;
    struct Arr {
        int cnt;
        short x[2048];
        short y[2048];
    };
    static constexpr Arr make() {
        Arr r{};
        r.cnt = 0;
        for (int p = 1; p < P2; p <<= 1)
            for (int k = p; k >= 1; k >>= 1)
                for (int j = k % p; j + k < P2; j += 2 * k)
                    for (int i = 0; i < k; ++i)
                        if (i + j + k < N && (i + j) / (2 * p) == (i + j + k) / (2 * p)) {
                            r.x[r.cnt] = (short)(i + j);
                            r.y[r.cnt] = (short)(i + j + k);
                            ++r.cnt;
                        }
        return r;
    }
    static constexpr Arr pairs = make();
};

template <int N, class CAS, int... C>
__device__ __forceinline__ void batcher_apply(CAS& cas, std::integer_sequence<int, C...>) {
    (cas(std::integral_constant<int, BatcherPairs<N>::pairs.x[C]>{},
         std::integral_constant<int, BatcherPairs<N>::pairs.y[C]>{}),
     ...);
}

template <int N, class CAS>
__device__ __forceinline__ void batcher_network(CAS&& cas) {
    batcher_apply<N>(cas, std::make_integer_sequence<int, BatcherPairs<N>::pairs.cnt>{});
}

// Sort IT keys held by one thread (the leaves and the in-thread levels).
// Keys-only u32/i32 (stability unobservable) use Batcher's network with
// min/max; the stable variants run it on (key, index) pairs.
template <class K, int IT, bool V>
__device__ __forceinline__ void thread_sort(uint32_t (&k)[IT], uint32_t (&ix)[IT]) {
    if constexpr (!V && !K::kNeedStable) {
        batcher_network<IT>([&](auto x, auto y) {
            constexpr int X = decltype(x)::value, Y = decltype(y)::value;
            const uint32_t lo = K::mn(k[X], k[Y]);
            const uint32_t hi = K::mx(k[X], k[Y]);
            k[X] = lo;
            k[Y] = hi;
        });
    } else {
        // Stable: the same network on (key, tile-local index) pairs, ordered
        // lexicographically; indices are distinct, so the order is total and
        // the result is the stable order of the keys.
        batcher_network<IT>([&](auto x, auto y) {
            constexpr int X = decltype(x)::value, Y = decltype(y)::value;
            const bool sw = K::lt(k[Y], k[X]) | (!K::lt(k[X], k[Y]) & (ix[Y] < ix[X]));
            const uint32_t klo = sw ? k[Y] : k[X], khi = sw ? k[X] : k[Y];
            const uint32_t ilo = sw ? ix[Y] : ix[X], ihi = sw ? ix[X] : ix[Y];
            k[X] = klo;
            k[Y] = khi;
            ix[X] = ilo;
            ix[Y] = ihi;
        });
    }
}

// ------------------------------------------------------- TMA bulk copies
// 1-D bulk copies (cp.async.bulk, SASS UBLKCP) between global and shared
// memory, completion tracked by an mbarrier transaction count (loads) or a
// bulk group (stores).  Addresses and sizes must be multiples of 16 bytes.
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t phase) {
    uint32_t done;
    do {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(done)
            : "r"(bar), "r"(phase)
            : "memory");
    } while (!done);
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes,
                                         uint32_t bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        ::"r"(dst), "l"(src), "r"(bytes), "r"(bar)
        : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, uint32_t src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst),
                 "r"(src), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_commit_and_wait_read() {
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
// Generic-proxy shared-memory writes -> visible to the async proxy (bulk store).
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// Store a shared tile to global memory.  Element e of the tile sits at shared
// word e + h and goes to dst[e], where h = (dst - 16-byte-aligned base) in
// words, so both sides of the bulk copy are congruent mod 16 bytes: the
// 16-byte body leaves by one TMA bulk copy issued by thread 0, the < 4-word
// head and tail by plain stores.  Caller: every thread has written its part,
// then fence_proxy_async_smem(); __syncthreads().
__device__ __forceinline__ void store_tile(uint32_t* __restrict__ dst, const uint32_t* s, int h,
                                           int count) {
#ifdef DC_NO_TMA_STORE   // sanitizer builds: compute-sanitizer initcheck does not track TMA writes
    for (int e = threadIdx.x; e < count; e += blockDim.x) dst[e] = s[h + e];
    return;
#endif
    const int head = min(count, (4 - h) & 3);              // words before the aligned body
    const int body = (count - head) & ~3;
    if (threadIdx.x == 0 && body > 0) {
        bulk_s2g(dst + head, smem_addr(s + h + head), 4u * body);
        bulk_commit_and_wait_read();
    }
    const int t = threadIdx.x;
    if (t < head) dst[t] = s[h + t];
    const int tail0 = head + body;
    if (t < count - tail0) dst[tail0 + t] = s[h + tail0 + t];
}

// ------------------------------------- first merge level by warp shuffles
// Keys-only: after the in-register network every thread holds one sorted run
// of IT keys; threads 2t and 2t+1 (lanes of one warp) merge theirs without
// shared memory.  The bitonic split min(A[j], B[IT-1-j]) / max(...) gives the
// lower / upper IT keys as bitonic sequences; the odd lane works on bit
// complements (~x reverses the order), so both lanes run the same
// instructions: exchange by one shuffle per key, take the minimum, sort the
// resulting ascending-then-descending sequence with a bitonic merge network
// (padded to a power of two with virtual minima that never cost an
// instruction, generated at compile time), and the odd lane un-complements and
// reverses.  Replaces one shared-memory level (~5 wavefronts per 32 keys:
// store, co-rank and conflicted merge loads) by one shuffle per key plus ALU.
template <int N>
struct BitonicPadNet {
    static constexpr int P2 = (N <= 1) ? 1 : (N <= 2) ? 2 : (N <= 4) ? 4 : (N <= 8) ? 8
                            : (N <= 16) ? 16 : (N <= 32) ? 32 : (N <= 64) ? 64 : 128;
    struct Arr {
        int cnt;
        short a[1024];
        short b[1024];
        short fin[128];   // fin[k]: register holding the k-th smallest after the network
    };
    static constexpr Arr make() {
        Arr r{};
        int map[P2] = {};
        bool pad[P2] = {};
        for (int p = 0; p < P2; ++p) { map[p] = p < N ? p : -1; pad[p] = p >= N; }
        r.cnt = 0;
        for (int d = P2 / 2; d >= 1; d /= 2)
            for (int i = 0; i < P2; ++i) {
                if (i & d) continue;
                const int j = i + d;
                if (pad[i] && pad[j]) continue;
                if (pad[j]) {          // j holds a virtual minimum: it moves to i for free
                    map[j] = map[i]; map[i] = -1; pad[i] = true; pad[j] = false;
                    continue;
                }
                if (pad[i]) continue;  // i already holds the minimum
                r.a[r.cnt] = (short)map[i];
                r.b[r.cnt] = (short)map[j];
                ++r.cnt;
            }
        for (int k = 0; k < N; ++k) r.fin[k] = (short)map[P2 - N + k];
        return r;
    }
    static constexpr Arr net = make();
};

template <int N, class F, int... C>
__device__ __forceinline__ void bitonic_pad_apply(F& f, std::integer_sequence<int, C...>) {
    (f(std::integral_constant<int, BitonicPadNet<N>::net.a[C]>{},
       std::integral_constant<int, BitonicPadNet<N>::net.b[C]>{}),
     ...);
}

template <int N, int... J>
__device__ __forceinline__ void bitonic_pad_final(uint32_t (&s)[N], const uint32_t (&u)[N],
                                                  std::integer_sequence<int, J...>) {
    ((s[J] = u[BitonicPadNet<N>::net.fin[J]]), ...);
}

template <int IT, class K>
__device__ __forceinline__ void merge_level_shfl(uint32_t (&k)[IT]) {
    const uint32_t m = (threadIdx.x & 1) ? 0xFFFFFFFFu : 0u;
    const bool odd = threadIdx.x & 1;
    uint32_t u[IT];
#pragma unroll
    for (int j = 0; j < IT; ++j) u[j] = (odd ? k[IT - 1 - j] : k[j]) ^ m;
#pragma unroll
    for (int j = 0; j < IT; ++j) {
        const uint32_t r = __shfl_xor_sync(0xffffffffu, u[j], 1) ^ 0xFFFFFFFFu;
        u[j] = K::mn(u[j], r);
    }
    auto cas = [&](auto a, auto b) {
        constexpr int A = decltype(a)::value, B = decltype(b)::value;
        const uint32_t lo = K::mn(u[A], u[B]), hi = K::mx(u[A], u[B]);
        u[A] = lo;
        u[B] = hi;
    };
    bitonic_pad_apply<IT>(cas, std::make_integer_sequence<int, BitonicPadNet<IT>::net.cnt>{});
    uint32_t s[IT];
    bitonic_pad_final<IT>(s, u, std::make_integer_sequence<int, IT>{});
#pragma unroll
    for (int j = 0; j < IT; ++j) k[j] = (odd ? s[IT - 1 - j] : s[j]) ^ m;
}

// ------------------------------------------- keys-only bitonic merge levels
// Keys-only u32/i32 (equal keys are identical bit patterns, so which copy of
// an equal key is emitted first is unobservable): every B run is stored
// DESCENDING after its ascending A run, so each pair is a bitonic sequence.
// A thread merges upward from the front of A and downward from the end of
// the pair (B's smallest).  When one run is exhausted, its pointer walks
// into the other run from that run's LARGEST end, so the value it reads is
// >= every element still pending and the plain comparison "b < a" keeps
// selecting the right side: no bounds checks, one tracked pointer.
// r02b: NK1 1.866 -> 1.814 ms per 2^28 u32 sort (5.90 -> 5.85 ms per step);
// 0 runs level 0 in shared memory like the others.
#ifndef DC_NK1_SHFL_L0
#define DC_NK1_SHFL_L0 1
#endif
template <int NT, int IT, class K>
__device__ __forceinline__ void merge_levels_bitonic(uint32_t (&k)[IT], uint32_t* sk) {
    constexpr int TILE = NT * IT;
    const int tid = threadIdx.x;
    const uint32_t SK = smem_addr(sk);
#ifndef DC_NK1_STOPW   // measurement knob only: stop the merge levels below this width
#define DC_NK1_STOPW (1 << 30)
#endif
    // w = IT * 2^lg at every level: the run index, the pair's thread group
    // and the diagonal are shifts and masks (runtime divisions by w compiled
    // to ~20-instruction float sequences, ~4 % of NK1's issue slots in r01)
    int lg = 0;
    int w0 = IT;
#if DC_NK1_SHFL_L0
    if (TILE >= 2 * IT) {            // level 0 (runs of IT -> 2 IT) without shared memory
        merge_level_shfl<IT, K>(k);
        w0 = 2 * IT;
        lg = 1;
    }
#endif
#pragma unroll 1
    for (int w = w0; w < TILE && w < DC_NK1_STOPW; w *= 2, ++lg) {
        // Levels whose pairs fit in one warp (2w <= 32*IT) only touch that
        // warp's own region: a warp barrier suffices and warps drift apart
        // (search / merge / write phases overlap across warps).
        const bool warp_local = 2 * w <= 32 * IT;
        if (warp_local) __syncwarp(); else __syncthreads();
        {   // write this thread's IT ascending keys: A runs ascending, B runs descending
            const int pos = tid * IT;
            const int r = tid >> lg;                      // run index at width w
            const int o = pos - r * w;                    // offset inside the run
            const int pr = (r >> 1) * (2 * w);            // pair start
            if ((r & 1) == 0) {
#pragma unroll
                for (int j = 0; j < IT; ++j) sk[pr + o + j] = k[j];
            } else {
#pragma unroll
                for (int j = 0; j < IT; ++j) sk[pr + 2 * w - 1 - o - j] = k[j];
            }
        }
        if (warp_local) __syncwarp(); else __syncthreads();
        const int s = (tid >> (lg + 1)) * (2 * w);        // pair start (2^(lg+1) threads per pair)
        const int diag = (tid & ((2 << lg) - 1)) * IT;
        // co-rank: A[m] at s + m, B[diag-1-m] at s + 2w - 1 - (diag-1-m) = s + 2w - diag + m
        const uint32_t Ab = SK + 4u * s, Bb = SK + 4u * (s + 2 * w - diag);
        int lo = max(0, diag - w), hi = min(diag, w);
        while (lo < hi) {
            const int m = (lo + hi) >> 1;
            if (!K::lt(lds(Bb + 4u * m), lds(Ab + 4u * m))) lo = m + 1;
            else hi = m;
        }
        // heads: A[lo] ascending pointer, B[diag-lo] at s + 2w - 1 - (diag - lo), descending
        uint32_t ai = Ab + 4u * lo;
        const uint32_t bi0 = SK + 4u * (s + 2 * w - 1 - (diag - lo));
        const uint32_t D = ai - bi0;                      // ai - bi grows by 4 per output
        uint32_t a = lds(ai), b = lds(bi0);
#pragma unroll
        for (int j = 0; j < IT; ++j) {
            const bool p = K::lt(b, a);                   // take B
            k[j] = p ? b : a;
            if (!p) ai += 4u;
            const uint32_t bi = ai - D - 4u * (j + 1);
            const uint32_t v = lds(p ? bi : ai);
            if (p) b = v; else a = v;
        }
    }
}

// ------------------------------------------------------------------ NK1
// One CTA sorts one tile of TILE = NT*IT keys (the last tile may be partial:
// it is padded with K::kPad, which sorts after every real key because every
// step is stable and the pads sit at the highest positions).
//   1. one TMA bulk copy brings the tile into shared memory; thread t then
//      reads its IT consecutive keys (conflict-free: IT is odd);
//   2. leaves + the levels inside a thread: in-register network;
//   3. levels with runs IT .. TILE/2: merge-path in shared memory, each
//      thread merging IT outputs serially;
//   4. the sorted tile leaves by one TMA bulk store.
// With values (V): the merges carry the tile-local index of every key, and
// the values are gathered by index at the end.
// Key-value NK1: the values are loaded after the last merge level, into the
// index region, so a CTA needs two tile regions instead of three (256 x 33:
// 67.6 KB, three CTAs per SM instead of two): NK1 3.33 -> 2.87 ms per 2^28
// key-value sort (r02b).  0 loads them with the keys into a third region.
#ifndef DC_NK1_KV_LATE
#define DC_NK1_KV_LATE 1
#endif
template <int NT, int IT, class K, bool V>
__global__ void __launch_bounds__(NT)
nk1_blocksort(const uint32_t* __restrict__ in_k, const uint32_t* __restrict__ in_v,
              uint32_t* __restrict__ out_k, uint32_t* __restrict__ out_v, long long n) {
    static_assert(IT % 2 == 1, "odd items per thread keep the blocked layout conflict-free");
    constexpr int TILE = NT * IT;
    static_assert(TILE % 4 == 0, "tile must be a whole number of 16-byte chunks");
    constexpr int TW = tile_words(TILE, 0);
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* sk = smem;              // [TW] keys
    uint32_t* si = smem + TW;         // [TW] tile-local indices, then gathered values (V)
    // [TW] values by original position (V).  DC_NK1_KV_LATE: the values arrive
    // after the last merge level, into the index region (the indices are in
    // registers by then), so the CTA needs two regions instead of three.
    uint32_t* sv = DC_NK1_KV_LATE ? si : smem + 2 * TW;
    __shared__ __align__(8) uint64_t bar;
    const uint32_t SK = smem_addr(sk);
    const uint32_t BAR = smem_addr(&bar);
    constexpr uint32_t SI_OFF = TW * 4;

    const int tid = threadIdx.x;
    const long long base = (long long)blockIdx.x * TILE;
    const int count = (int)min((long long)TILE, n - base);
    const int body = count & ~3;       // 16-byte part moved by TMA

    // ---- 1. load
    constexpr bool kEarlyV = V && !DC_NK1_KV_LATE;
    if (tid == 0) {
        mbar_init(BAR, 1);
        mbar_arrive_expect_tx(BAR, 4u * body * (kEarlyV ? 2 : 1));
        if (body > 0) {
            bulk_g2s(SK, in_k + base, 4u * body, BAR);
            if (kEarlyV) bulk_g2s(smem_addr(sv), in_v + base, 4u * body, BAR);
        }
    }
    for (int e = body + tid; e < TILE; e += NT) {   // ragged tail + pads
        sk[e] = e < count ? in_k[base + e] : K::kPad;
        if (kEarlyV) sv[e] = e < count ? in_v[base + e] : 0u;
    }
    __syncthreads();                  // barrier init + tail visible
    mbar_wait(BAR, 0);
    uint32_t k[IT];
    uint32_t ix[IT];
#pragma unroll
    for (int j = 0; j < IT; ++j) {
        k[j] = sk[tid * IT + j];
        ix[j] = tid * IT + j;
    }

    // ---- 2. leaves + in-thread levels
#ifndef DC_NK1_NOREG   // measurement knob only
    thread_sort<K, IT, V>(k, ix);
#endif

    // ---- 3. shared-memory merge levels: run width w -> 2w
    if constexpr (!V && !K::kNeedStable) {
        merge_levels_bitonic<NT, IT, K>(k, sk);
    } else {
        int lg = 0;                                    // w = IT * 2^lg (shifts, not divisions)
#pragma unroll 1
        for (int w = IT; w < TILE; w *= 2, ++lg) {
            __syncthreads();
#pragma unroll
            for (int j = 0; j < IT; ++j) {
                sk[tid * IT + j] = k[j];
                if (V) si[tid * IT + j] = ix[j];
            }
            __syncthreads();
            const int s = (tid >> (lg + 1)) * (2 * w);   // pair start (2^(lg+1) threads per pair)
            const int diag = (tid & ((2 << lg) - 1)) * IT;
            const uint32_t A = SK + 4u * s, B = A + 4u * w;
            const int i = corank_smem<K>(A, w, B, w, diag);
            uint32_t src[IT];
            serial_merge<K, IT, V>(A + 4u * i, B, B + 4u * (diag - i), B + 4u * w, k, src);
            if (V) {
#pragma unroll
                for (int j = 0; j < IT; ++j) ix[j] = lds(src[j] + SI_OFF);
            }
        }
    }

    // ---- 4. store: blocked write into shared memory, one bulk store
    if (V && DC_NK1_KV_LATE) fence_proxy_async_smem();   // index writes before the TMA refill
    __syncthreads();
    if constexpr (V && DC_NK1_KV_LATE) {
        // the values by original position into the (now free) index region
        if (tid == 0) {
            mbar_arrive_expect_tx(BAR, 4u * body);
            if (body > 0) bulk_g2s(smem_addr(sv), in_v + base, 4u * body, BAR);
        }
        for (int e = body + tid; e < TILE; e += NT) sv[e] = e < count ? in_v[base + e] : 0u;
#pragma unroll
        for (int j = 0; j < IT; ++j) sk[tid * IT + j] = k[j];
        __syncthreads();                  // barrier phase 1 armed, tail written
        mbar_wait(BAR, 1);
        uint32_t vv[IT];
#pragma unroll
        for (int j = 0; j < IT; ++j) vv[j] = sv[ix[j]];   // gather the values by index
        __syncthreads();
#pragma unroll
        for (int j = 0; j < IT; ++j) si[tid * IT + j] = vv[j];
    } else {
#pragma unroll
        for (int j = 0; j < IT; ++j) {
            sk[tid * IT + j] = k[j];
            if (V) si[tid * IT + j] = sv[ix[j]];    // gather the values by index
        }
    }
    fence_proxy_async_smem();
    __syncthreads();
    store_tile(out_k + base, sk, 0, count);
    if (V) store_tile(out_v + base, si, 0, count);
}

// ------------------------------------------ NK1 + cluster levels (f2)
// SURVEY f2's cluster / distributed-shared-memory levels (keys-only u32/i32):
// a cluster of CS CTAs (CS = 2, 4, 8 or 16, a launch attribute) sorts CS
// adjacent tiles exactly like nk1_blocksort, then runs log2(CS) more merge
// levels on chip.  At cluster level g (runs of g tiles -> 2g tiles), CTA r of
// a group pair [p0, p0 + 2g) produces the outputs [(r - p0)*TILE, +TILE) of
// merge(A, B), A = tiles p0 .. p0+g-1, B = the next g tiles, each tile sorted
// in its own CTA's shared memory:
//   1. two warps find the co-ranks c(d0), c(d0 + TILE) of its output range by
//      33-ary warp searches through the cluster window (ld.shared::cluster);
//   2. every thread gathers its share of the TILE inputs A[c0, c1) and
//      B[d0 - c0, d0 + TILE - c1) from the owning CTAs (coalesced DSMEM loads
//      into registers);
//   3. a cluster barrier (every read of every tile done), the inputs go to the
//      CTA's own shared memory as two sorted runs, and one local merge-path
//      level (co-rank + serial merge) produces the CTA's TILE outputs.
// The fused runs are CS tiles wide, so log2(CS) global levels fewer remain.
// Every level is the stable merge of adjacent runs (A wins ties), i.e. Alg 7's
// combine; for keys-only sorts the result is the sorted multiset.
// Measured: a cluster level costs more than a global level
// at 2^28 but far less than one at small n, where every global level is a
// latency-bound launch; the planner's cluster rule (dc_api.cu) picks CS.
// (A first prototype merged straight out of the partner's shared memory --
// every serial-merge step a DSMEM load -- and cost 0.98 ms per 2^28 level.)
__device__ __forceinline__ uint32_t ldcl(uint32_t addr) {   // shared::cluster address
    uint32_t v;
    asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
}
__device__ __forceinline__ uint32_t cluster_map(uint32_t local_addr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(local_addr), "r"(rank));
    return r;
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cluster_size() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// Element i of a run of g tiles starting at cluster rank `first` (tile t of
// the run lives in CTA first + t, word i mod TILE of its tile buffer SK).
template <int TILE>
__device__ __forceinline__ uint32_t run_at(uint32_t SK, uint32_t first, int i) {
    const int t = i / TILE;
    return ldcl(cluster_map(SK + 4u * (uint32_t)(i - t * TILE), first + (uint32_t)t));
}

// c(d) = #A among the first d outputs of merge(A, B), both runs of width W
// (A wins ties), by a 33-ary search of one warp through the cluster window:
// P(q) = "q <= c" = A[q - 1] <= B[d - q] is monotone, probes that hold are a
// prefix.  Returns c in every lane.
template <class K, int TILE>
__device__ __forceinline__ int cluster_corank(uint32_t SK, uint32_t fa, uint32_t fb, int W, int d) {
    const int lane = threadIdx.x & 31;
    int lo = max(0, d - W), hi = min(d, W);
    while (hi > lo) {
        const int step = (hi - lo + 31) >> 5;       // probes lo + (l + 1) * step reach hi
        const int q = lo + (lane + 1) * step;
        bool ok = false;
        if (q <= hi) ok = !K::lt(run_at<TILE>(SK, fb, d - q), run_at<TILE>(SK, fa, q - 1));
        const int nt = __popc(__ballot_sync(0xffffffffu, ok));
        const int nlo = lo + nt * step;
        hi = min(hi, lo + (nt + 1) * step - 1);
        lo = nlo;
    }
    return lo;
}

template <int NT, int IT, class K>
__global__ void __launch_bounds__(NT)
nk1_blocksort_cl(const uint32_t* __restrict__ in_k, uint32_t* __restrict__ out_k, long long n) {
    static_assert(IT % 2 == 1, "odd items per thread keep the blocked layout conflict-free");
    static_assert(!K::kNeedStable, "keys-only");
    static_assert(NT >= 64, "two warps search the co-ranks");
    constexpr int TILE = NT * IT;
    extern __shared__ __align__(16) uint32_t smem[];
    uint32_t* sk = smem;              // [TILE + slack]
    __shared__ __align__(8) uint64_t bar;
    __shared__ int s_c[2];
    const uint32_t SK = smem_addr(sk);
    const uint32_t BAR = smem_addr(&bar);
    const int tid = threadIdx.x;
    const uint32_t rank = cluster_rank(), CS = cluster_size();
    const long long base = (long long)blockIdx.x * TILE;
    const int count = (int)max(0LL, min((long long)TILE, n - base));
    const int body = count & ~3;

    if (tid == 0) {
        mbar_init(BAR, 1);
        mbar_arrive_expect_tx(BAR, 4u * body);
        if (body > 0) bulk_g2s(SK, in_k + base, 4u * body, BAR);
    }
    for (int e = body + tid; e < TILE; e += NT) sk[e] = e < count ? in_k[base + e] : K::kPad;
    __syncthreads();
    mbar_wait(BAR, 0);
    uint32_t k[IT];
    uint32_t ix[IT];
#pragma unroll
    for (int j = 0; j < IT; ++j) k[j] = sk[tid * IT + j];
    thread_sort<K, IT, false>(k, ix);
    merge_levels_bitonic<NT, IT, K>(k, sk);      // this tile sorted, in registers

#pragma unroll 1
    for (uint32_t g = 1; g < CS; g <<= 1) {
        __syncthreads();
#pragma unroll
        for (int j = 0; j < IT; ++j) sk[tid * IT + j] = k[j];
        cluster_sync_all();                      // every CTA's run piece visible
        const uint32_t p0 = rank & ~(2 * g - 1);
        const int W = (int)g * TILE;
        const int d0 = (int)(rank - p0) * TILE;
        if (tid < 64) {
            const int c = cluster_corank<K, TILE>(SK, p0, p0 + g, W, d0 + (tid >> 5) * TILE);
            if ((tid & 31) == 0) s_c[tid >> 5] = c;
        }
        __syncthreads();
        const int c0 = s_c[0], c1 = s_c[1];
        const int a = c1 - c0;                   // A elements of this CTA's outputs
        const int b0 = d0 - c0;                  // first B element
#pragma unroll
        for (int j = 0; j < IT; ++j) {
            const int e = j * NT + tid;          // input e of TILE: A part, then B part
            k[j] = e < a ? run_at<TILE>(SK, p0, c0 + e) : run_at<TILE>(SK, p0 + g, b0 + e - a);
        }
        cluster_sync_all();                      // every read of every tile done
#pragma unroll
        for (int j = 0; j < IT; ++j) sk[j * NT + tid] = k[j];
        __syncthreads();
        const int d = tid * IT;
        const int i1 = corank_smem<K>(SK, a, SK + 4u * a, TILE - a, d);
        uint32_t srcs[IT];
        serial_merge<K, IT, false>(SK + 4u * i1, SK + 4u * a, SK + 4u * (a + d - i1),
                                   SK + 4u * TILE, k, srcs);
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < IT; ++j) sk[tid * IT + j] = k[j];
    fence_proxy_async_smem();
    __syncthreads();
    // the cluster's real keys come first (pads are maximum keys)
    const long long cbase = base - (long long)rank * TILE;
    const long long tot = max(0LL, min((long long)CS * TILE, n - cbase));
    const int cnt = (int)max(0LL, min((long long)TILE, tot - (long long)rank * TILE));
    if (cnt > 0) store_tile(out_k + base, sk, 0, cnt);
}

// ------------------------------------------------------------------ NK2
// Geometry of one merge level over [org, end) of a buffer: pairs of adjacent
// runs (A of width wa, then B of width wb) with stride wa + wb starting at
// org; the last pair may be short.  The breadth-first sort uses org = 0 and
// wa = wb = w; the local G-way merge of the multi-GPU path merges one pair of
// arbitrary lengths at an arbitrary offset per launch.  Indices are absolute
// (the buffer base stays 16-byte aligned for TMA).
struct PairGeom {
    long long org, wa, wb, end;
    int tpg;   // output tiles per pair: ceil((wa + wb) / tout) (the last one short)
    // Tile j: absolute pair start s, run lengths, tile output range [dd0, dd1)
    // relative to s (empty when dd0 >= a_len + b_len: trailing tiles of a
    // short last pair).
    __device__ __forceinline__ void tile_of(int j, int tout, long long& s, long long& a_len,
                                            long long& b_len, long long& dd0,
                                            long long& dd1) const {
        const int p = j / tpg;
        s = org + (long long)p * (wa + wb);
        a_len = min(wa, end - s);
        b_len = max(0LL, min(wb, end - s - a_len));
        dd0 = (long long)(j - p * tpg) * tout;
        dd1 = min(dd0 + tout, a_len + b_len);
    }
};

// Co-rank of the first output of every merge tile (tile j: tile_of).
template <class K>
__global__ void nk2_partition(const uint32_t* __restrict__ src, PairGeom g, int tout,
                              int num_tiles, int* __restrict__ split) {
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= num_tiles) return;
    long long s, a_len, b_len, dd0, dd1;
    g.tile_of(j, tout, s, a_len, b_len, dd0, dd1);
    if (dd0 >= a_len + b_len) return;                 // empty tile
    split[j] = (int)corank_global<K>(src + s, a_len, src + s + a_len, b_len, dd0);
}

// First index in [a, b] where a monotone (true ... false) predicate on [a, b)
// is false (b if none), found by one warp: every round the 32 lanes evaluate
// f at 32 evenly spaced points (__ballot), shrinking the interval 33-fold.
template <class F>
__device__ __forceinline__ long long warp_first_false(long long a, long long b, F f) {
    const int lane = threadIdx.x & 31;
    while (a < b) {
        const long long span = b - a;
        const long long pos = a + ((lane + 1) * span) / 33;       // < b
        const unsigned fm = __ballot_sync(0xffffffffu, !f(pos));
        if (fm == 0) {
            a = a + (32 * span) / 33 + 1;
        } else {
            const int L = __ffs(fm) - 1;
            const long long posL = a + ((L + 1) * span) / 33;
            const long long posP = L > 0 ? a + (L * span) / 33 : a - 1;
            b = posL;
            a = posP + 1;
        }
    }
    return a;
}

// NK2, warp per tile (small, L2-resident inputs): the same co-rank found by a
// 33-ary warp search -- ~log33(w) dependent rounds instead of log2(w).  Used
// when the array fits in L2, where the extra probes cost no HBM traffic.
template <class K>
__global__ void nk2_partition_warp(const uint32_t* __restrict__ src, PairGeom g, int tout,
                                   int num_tiles, int* __restrict__ split) {
    const int j = (int)(((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    if (j >= num_tiles) return;                       // warp-uniform
    long long s, a_len, b_len, diag, dd1;
    g.tile_of(j, tout, s, a_len, b_len, diag, dd1);
    if (diag >= a_len + b_len) return;                // empty tile
    const uint32_t* A = src + s;
    const uint32_t* B = src + s + a_len;
    const long long lo = max(0LL, diag - b_len), hi = min(diag, a_len);
    const long long c = warp_first_false(lo, hi, [&](long long m) {
        return !K::lt(__ldg(B + (diag - 1 - m)), __ldg(A + m));
    });
    if ((threadIdx.x & 31) == 0) split[j] = (int)c;
}

// ------------------------------------------------------------------ NK3
// Stage global elements [g0, g1) (any alignment) into shared memory at word
// offset `off` + (g0 & 3): TMA copies the 16-byte-aligned superset that lies
// below n4 = n & ~3; the caller's threads load the rest (< 4 words past n4).
__device__ __forceinline__ uint32_t piece_bytes(long long g0, long long g1, long long n4) {
    const long long al0 = g0 & ~3LL;
    long long al1 = (g1 + 3) & ~3LL;
    if (al1 > n4) al1 = n4;
    return al1 > al0 ? (uint32_t)(4 * (al1 - al0)) : 0u;
}
__device__ __forceinline__ void stage_piece(const uint32_t* __restrict__ g, long long g0,
                                            long long g1, long long n4, uint32_t dst_off,
                                            uint32_t sbase, uint32_t bar) {
    const uint32_t bytes = piece_bytes(g0, g1, n4);
    if (bytes) bulk_g2s(sbase + 4u * dst_off, g + (g0 & ~3LL), bytes, bar);
}

// One output tile of the merge of A = src[a0, a0+na) and B = src[b0, b0+nb)
// (total = na + nb <= NT*IT outputs) written to dst[o0, o0+total).  The
// pieces are staged in shared memory by TMA, each thread finds its own
// IT-output diagonal there and merges serially, and the tile leaves by one
// TMA bulk store.  n bounds the readable part of src.
//
// A and B may live in different buffers (e.g. a peer GPU's memory, read over
// NVLink by the multi-GPU merge): src_a / src_b are 16-byte-aligned buffer
// bases, na_bound / nb_bound their readable lengths, a0 / b0 offsets in them.
template <int NT, int IT, class K, bool V>
__device__ __forceinline__ void merge_tile(const uint32_t* __restrict__ src_ka,
                                           const uint32_t* __restrict__ src_va, long long n_a,
                                           long long a0, int na,
                                           const uint32_t* __restrict__ src_kb,
                                           const uint32_t* __restrict__ src_vb, long long n_b,
                                           long long b0, int nb,
                                           uint32_t* __restrict__ dst_k,
                                           uint32_t* __restrict__ dst_v, long long o0,
                                           uint32_t* sk, uint32_t* sv, uint32_t BAR) {
    constexpr int TOUT = NT * IT;
    constexpr int TW = tile_words(TOUT, IT + 16);
    constexpr uint32_t SV_OFF = TW * 4;
    const uint32_t SK = smem_addr(sk), SV = smem_addr(sv);
    const int tid = threadIdx.x;
    const int total = na + nb;
    const int fa = (int)(a0 & 3), fb = (int)(b0 & 3);
    const int ob = (fa + na + 1 + 3) & ~3;             // B region word offset (16 B aligned)
    const uint32_t A = SK + 4u * fa, B = SK + 4u * (ob + fb);
    const long long a4 = n_a & ~3LL, b4 = n_b & ~3LL;

    if (tid == 0) {
        mbar_init(BAR, 1);
        const uint32_t bytes = piece_bytes(a0, a0 + na, a4) + piece_bytes(b0, b0 + nb, b4);
        mbar_arrive_expect_tx(BAR, bytes * (V ? 2 : 1));
        stage_piece(src_ka, a0, a0 + na, a4, 0, SK, BAR);
        stage_piece(src_kb, b0, b0 + nb, b4, ob, SK, BAR);
        if (V) {
            stage_piece(src_va, a0, a0 + na, a4, 0, SV, BAR);
            stage_piece(src_vb, b0, b0 + nb, b4, ob, SV, BAR);
        }
    }
    // elements at or beyond the aligned bound (only in the last pieces of a buffer)
    if (a0 + na > a4) {
        for (long long g = max(a0, a4) + tid; g < a0 + na; g += NT) {
            sk[fa + (g - a0)] = src_ka[g];
            if (V) sv[fa + (g - a0)] = src_va[g];
        }
    }
    if (b0 + nb > b4) {
        for (long long g = max(b0, b4) + tid; g < b0 + nb; g += NT) {
            sk[ob + fb + (g - b0)] = src_kb[g];
            if (V) sv[ob + fb + (g - b0)] = src_vb[g];
        }
    }
    __syncthreads();
    mbar_wait(BAR, 0);

    const int diag = tid * IT;
    uint32_t k[IT], src[IT], vv[IT];
    if (diag < total) {
        const int i = corank_smem<K>(A, na, B, nb, diag);
        serial_merge<K, IT, V>(A + 4u * i, A + 4u * na, B + 4u * (diag - i), B + 4u * nb, k,
                               src);
        if (V) {
#pragma unroll
            for (int q = 0; q < IT; ++q) vv[q] = lds(src[q] + SV_OFF);
        }
    }
    __syncthreads();
    const int h = (int)(o0 & 3);                       // output alignment shift
    if (diag < total) {
#pragma unroll
        for (int q = 0; q < IT; ++q) {
            sk[h + diag + q] = k[q];
            if (V) sv[h + diag + q] = vv[q];
        }
    }
    fence_proxy_async_smem();
    __syncthreads();
    store_tile(dst_k + o0, sk, h, total);
    if (V) store_tile(dst_v + o0, sv, h, total);
}

// One merge level (Alg 7 lines 3-5): CTA j produces merged positions
// [j*TOUT, (j+1)*TOUT) of the pair that contains them, in place in dst.
template <int NT, int IT, class K, bool V>
__global__ void __launch_bounds__(NT)
nk3_merge(const uint32_t* __restrict__ src_k, const uint32_t* __restrict__ src_v,
          uint32_t* __restrict__ dst_k, uint32_t* __restrict__ dst_v,
          const int* __restrict__ split, PairGeom g) {
    static_assert(IT % 2 == 1, "odd items per thread keep the blocked layout conflict-free");
    constexpr int TOUT = NT * IT;
    constexpr int TW = tile_words(TOUT, IT + 16);
    extern __shared__ __align__(16) uint32_t smem[];
    __shared__ __align__(8) uint64_t bar;
    const int j = blockIdx.x;
    long long s, a_len, b_len, dd0, dd1;
    g.tile_of(j, TOUT, s, a_len, b_len, dd0, dd1);
    if (dd0 >= a_len + b_len) return;                 // empty tile (whole CTA)
    const int i0 = split[j];
    const int i1 = (dd1 == a_len + b_len) ? (int)a_len : split[j + 1];
    const int na = i1 - i0;
    const int nb = (int)(dd1 - dd0) - na;
    merge_tile<NT, IT, K, V>(src_k, src_v, g.end, s + i0, na, src_k, src_v, g.end,
                             s + a_len + (dd0 - i0), nb, dst_k, dst_v, s + dd0, smem,
                             smem + TW, smem_addr(&bar));
}

// One merge level with the partition fused in (L2-resident sorts, where a
// level is a few microseconds and a separate NK2 launch is a large share):
// warps 0 and 1 of CTA j find the co-ranks of the tile's first and last+1
// outputs with 33-ary warp searches (a few dependent L2 round trips), then
// the CTA merges its tile as nk3_merge does.
template <int NT, int IT, class K, bool V>
__global__ void __launch_bounds__(NT)
nk3_merge_sp(const uint32_t* __restrict__ src_k, const uint32_t* __restrict__ src_v,
             uint32_t* __restrict__ dst_k, uint32_t* __restrict__ dst_v, PairGeom g) {
    static_assert(NT >= 64, "two searching warps");
    constexpr int TOUT = NT * IT;
    constexpr int TW = tile_words(TOUT, IT + 16);
    extern __shared__ __align__(16) uint32_t smem[];
    __shared__ __align__(8) uint64_t bar;
    __shared__ int cr[2];
    const int j = blockIdx.x;
    long long s, a_len, b_len, dd0, dd1;
    g.tile_of(j, TOUT, s, a_len, b_len, dd0, dd1);
    if (dd0 >= a_len + b_len) return;                 // empty tile (whole CTA)
    const int warp = threadIdx.x >> 5;
    if (warp < 2) {
        const long long diag = warp == 0 ? dd0 : dd1;
        const uint32_t* A = src_k + s;
        const uint32_t* B = src_k + s + a_len;
        const long long lo = max(0LL, diag - b_len), hi = min(diag, a_len);
        const long long c = warp_first_false(lo, hi, [&](long long m) {
            return !K::lt(__ldg(B + (diag - 1 - m)), __ldg(A + m));
        });
        if ((threadIdx.x & 31) == 0) cr[warp] = (int)c;
    }
    __syncthreads();
    const int i0 = cr[0], i1 = cr[1];
    const int na = i1 - i0;
    const int nb = (int)(dd1 - dd0) - na;
    merge_tile<NT, IT, K, V>(src_k, src_v, g.end, s + i0, na, src_k, src_v, g.end,
                             s + a_len + (dd0 - i0), nb, dst_k, dst_v, s + dd0, smem,
                             smem + TW, smem_addr(&bar));
}

// ------------------------------------------- merges of separately stored runs
// The first round of the multi-GPU G-way merge reads its two runs straight
// from the sorted shards of two (peer) GPUs -- the exchange fused into the
// merge, the NVLink reads overlapping the merge tile by tile.  A run is
// (buffer base, readable length, offset, length); bases are 16-byte aligned.

// Co-rank of every output tile of merge(A, B), one warp per tile (33-ary
// search: ~log33 of the run length dependent rounds of remote latency).
template <class K>
__global__ void nk2_partition_ab(const uint32_t* __restrict__ A, long long a_len,
                                 const uint32_t* __restrict__ B, long long b_len, int tout,
                                 int num_tiles, int* __restrict__ split) {
    const int j = (int)(((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    if (j >= num_tiles) return;                       // warp-uniform
    const long long diag = (long long)j * tout;
    const long long lo = max(0LL, diag - b_len), hi = min(diag, a_len);
    const long long c = warp_first_false(lo, hi, [&](long long m) {
        return !K::lt(__ldg(B + (diag - 1 - m)), __ldg(A + m));
    });
    if ((threadIdx.x & 31) == 0) split[j] = (int)c;
}

// Output tile j of merge(A, B) -> dst[o_off + j*TOUT, ...).
template <int NT, int IT, class K, bool V>
__global__ void __launch_bounds__(NT)
nk3_merge_ab(const uint32_t* __restrict__ ka, const uint32_t* __restrict__ va, long long a_bound,
             long long a_off, long long a_len, const uint32_t* __restrict__ kb,
             const uint32_t* __restrict__ vb, long long b_bound, long long b_off, long long b_len,
             uint32_t* __restrict__ dst_k, uint32_t* __restrict__ dst_v, long long o_off,
             const int* __restrict__ split) {
    constexpr int TOUT = NT * IT;
    constexpr int TW = tile_words(TOUT, IT + 16);
    extern __shared__ __align__(16) uint32_t smem[];
    __shared__ __align__(8) uint64_t bar;
    const long long d0 = (long long)blockIdx.x * TOUT;
    const long long d1 = min(d0 + TOUT, a_len + b_len);
    const int i0 = split[blockIdx.x];
    const int i1 = (d1 == a_len + b_len) ? (int)a_len : split[blockIdx.x + 1];
    const int na = i1 - i0;
    const int nb = (int)(d1 - d0) - na;
    merge_tile<NT, IT, K, V>(ka, va, a_bound, a_off + i0, na, kb, vb, b_bound,
                             b_off + (d0 - i0), nb, dst_k, dst_v, o_off + d0, smem, smem + TW,
                             smem_addr(&bar));
}

}  // namespace dc
