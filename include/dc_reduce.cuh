// dc_reduce.cuh -- generic O(1)-combine breadth-first divide and conquer.
//
// Header-only device template for any D&C whose combine is O(1) and
// associative (not necessarily commutative): T(n) = 2T(n/2) + O(1).  The
// paper's own example is the D&C sum (Alg 4; its GPU form Alg 5,
// P:L389-395, runs one kernel per level pairing a[id] with a[id+m]).  Here the
// levels are executed breadth-first but fused by locality, as NK4/NK5 do for
// max-subarray:
//   leaves + bottom levels : every thread folds a contiguous chunk left to right;
//   middle levels          : ordered warp-shuffle then cross-warp combines
//                            (lane i is the LEFT operand of lane i + d, so a
//                            non-commutative combine stays correct -- Alg 5's
//                            strided pairing is only valid for commutative ones);
//   top levels             : the last CTA to finish (atomic ticket) combines the
//                            per-CTA summaries in order.
// A monoid M provides
//   using In = <element type>;  using T = <summary type, trivially copyable>;
//   static __device__ T identity();
//   static __device__ T leaf(In x, long long i);          // base case at index i
//   static __device__ T combine(const T& l, const T& r);  // l immediately left of r
// and the caller provides `parts` (one T per CTA) and a zero-initialised
// `ticket`; the result is written to *out by the last CTA.  Launch with a grid
// of at most a few waves; NT threads per CTA (multiple of 32, <= 1024).
// Two kernels: breadth_first_reduce (plain loads, any element type) and
// breadth_first_reduce_tma (TMA-streamed warp segments, 4-byte elements;
// the library's dc_run_sum uses it).
#pragma once
#include <cstdint>

namespace dc {

template <class T>
__device__ __forceinline__ T reduce_shfl_down(const T& v, int off) {
    static_assert(sizeof(T) % 4 == 0, "summary must be a whole number of 32-bit words");
    T r;
    const int* s = reinterpret_cast<const int*>(&v);
    int* d = reinterpret_cast<int*>(&r);
#pragma unroll
    for (int q = 0; q < (int)(sizeof(T) / 4); ++q) d[q] = __shfl_down_sync(0xffffffffu, s[q], off);
    return r;
}

// Ordered combine of one summary per thread (thread order = segment order);
// the result is valid in thread 0.  red: NT/32 summaries of shared memory.
// The shuffle trees are branch-free: every lane combines with its partner at
// every level, and only lanes that are multiples of 2*off carry a meaningful
// summary into the next level (a conditional combine makes the following
// full-mask shuffles potentially divergent, and the compiler then guards each
// level with a WARPSYNC fallback).  M::combine must therefore be total: it
// also sees pairs of valid summaries in the wrong order, whose results are
// discarded.
template <class M, int NT>
__device__ __forceinline__ typename M::T reduce_block(typename M::T t, typename M::T* red) {
    using T = typename M::T;
    static_assert(NT % 32 == 0 && NT <= 1024, "block of whole warps");
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const T r = reduce_shfl_down(t, off);
        t = M::combine(t, r);   // branch-free: only lanes = 0 mod 2*off stay meaningful
    }
    if (lane == 0) red[warp] = t;
    __syncthreads();
    if (warp == 0) {
        t = lane < NT / 32 ? red[lane] : M::identity();
#pragma unroll
        for (int off = 1; off < NT / 32; off <<= 1) {
            const T r = reduce_shfl_down(t, off);
            t = M::combine(t, r);   // branch-free: only lanes = 0 mod 2*off stay meaningful
        }
    }
    __syncthreads();
    return t;
}

// Breadth-first O(1)-combine D&C over x[0..n): CTA c folds the contiguous
// tiles [c*nt/G, (c+1)*nt/G) of NT*C elements; thread t folds the contiguous
// chunk [t*C, t*C + C) of each tile.
template <class M, int NT, int C>
__global__ void __launch_bounds__(NT)
breadth_first_reduce(const typename M::In* __restrict__ x, long long n,
                     typename M::T* __restrict__ parts, unsigned int* __restrict__ ticket,
                     typename M::T* __restrict__ out) {
    using T = typename M::T;
    constexpr int TILE = NT * C;
    __shared__ T red[NT / 32];
    __shared__ bool am_last;
    const int tid = threadIdx.x;
    const long long ntiles = (n + TILE - 1) / TILE;
    const long long t0 = ntiles * blockIdx.x / gridDim.x;
    const long long t1 = ntiles * (blockIdx.x + 1) / gridDim.x;
    T acc = M::identity();
    for (long long tile = t0; tile < t1; ++tile) {
        const long long beg = tile * TILE + (long long)tid * C;
        T f = M::identity();
#pragma unroll 4
        for (int q = 0; q < C; ++q) {
            const long long e = beg + q;
            if (e < n) f = M::combine(f, M::leaf(__ldg(x + e), e));
        }
        f = reduce_block<M, NT>(f, red);
        if (tid == 0) acc = M::combine(acc, f);
    }
    if (tid == 0) {
        parts[blockIdx.x] = acc;
        __threadfence();
        am_last = atomicAdd(ticket, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!am_last) return;
    __threadfence();
    const int np = gridDim.x, per = (np + NT - 1) / NT;
    T a = M::identity();
    for (int q = tid * per; q < min(np, tid * per + per); ++q) {
        T v;
        const volatile int* src = reinterpret_cast<const volatile int*>(parts + q);
        int* dst = reinterpret_cast<int*>(&v);
#pragma unroll
        for (int w = 0; w < (int)(sizeof(T) / 4); ++w) dst[w] = src[w];   // L2-coherent
        a = M::combine(a, v);
    }
    a = reduce_block<M, NT>(a, red);
    if (tid == 0) {
        *out = a;
        *ticket = 0u;   // re-arm for the next launch
    }
}

// ------------------------------------------------------------------------
// breadth_first_reduce_tma: the same D&C with the data streamed by TMA.
// Every WARP owns one contiguous range of RW elements (RW a multiple of
// 32*L) and streams it in segments of 32*L elements, one 1-D bulk copy per
// segment into an S-stage shared-memory ring (mbarrier per warp and stage);
// lane l folds the L contiguous elements [l*L, (l+1)*L) of each segment
// (128-bit shared reads, bank-conflict free because L/4 is odd), an ordered
// shuffle tree combines the 32 lane summaries, lane 0 keeps the warp's running
// summary; warps, then CTAs (last CTA, atomic ticket), combine in order.
// Requirements: sizeof(In) == 4, x 16-byte aligned; launch with NT threads,
// breadth_first_reduce_tma_smem<NT, L, S>() bytes of dynamic shared memory
// (raise cudaFuncAttributeMaxDynamicSharedMemorySize above 48 KB) and a grid
// of at most one wave; RW = breadth_first_reduce_tma_rw<NT, L>(n, grid).
namespace rtma {
__device__ __forceinline__ uint32_t saddr(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void bar_init(uint32_t bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void bar_expect(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bar_wait(uint32_t bar, uint32_t phase) {
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
__device__ __forceinline__ void copy(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        ::"r"(dst), "l"(src), "r"(bytes), "r"(bar)
        : "memory");
}
__device__ __forceinline__ void fence_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
}  // namespace rtma

template <int NT, int L, int S>
constexpr size_t breadth_first_reduce_tma_smem() {
    return (size_t)S * NT * L * 4;
}
template <int NT, int L>
inline long long breadth_first_reduce_tma_rw(long long n, int grid) {
    const long long warps = (long long)grid * (NT / 32), seg = 32LL * L;
    return ((n + warps - 1) / warps + seg - 1) / seg * seg;
}

template <class M, int NT, int L, int S>
__global__ void __launch_bounds__(NT)
breadth_first_reduce_tma(const typename M::In* __restrict__ x, long long n, long long RW,
                         typename M::T* __restrict__ parts, unsigned int* __restrict__ ticket,
                         typename M::T* __restrict__ out) {
    using T = typename M::T;
    using In = typename M::In;
    static_assert(sizeof(In) == 4, "4-byte elements");
    static_assert(L % 4 == 0 && ((L / 4) & 1) == 1, "L/4 odd: conflict-free 128-bit reads");
    constexpr int NW = NT / 32, SEG = 32 * L;
    extern __shared__ __align__(16) unsigned char rtma_smem[];
    In* ring = reinterpret_cast<In*>(rtma_smem);               // [S][NW][SEG]
    __shared__ __align__(8) uint64_t bars[S][NW];
    __shared__ T red[NW];
    __shared__ bool am_last;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const long long wbeg = min(n, ((long long)blockIdx.x * NW + warp) * RW);
    const long long wend = min(n, wbeg + RW);
    const int nseg = (int)((wend - wbeg + SEG - 1) / SEG);
    if (lane == 0)
        for (int s = 0; s < S; ++s) rtma::bar_init(rtma::saddr(&bars[s][warp]));
    __syncwarp();
    auto seg_ptr = [&](int s) { return ring + (s * NW + warp) * SEG; };
    auto issue = [&](int k) {
        const int s = k % S;
        const long long g0 = wbeg + (long long)k * SEG;
        const int body = (int)min((long long)SEG, wend - g0) & ~3;
        const uint32_t bar = rtma::saddr(&bars[s][warp]);
        rtma::bar_expect(bar, 4u * body);
        if (body) rtma::copy(rtma::saddr(seg_ptr(s)), x + g0, 4u * body, bar);
    };
    if (lane == 0)
        for (int k = 0; k < S && k < nseg; ++k) issue(k);
    T acc = M::identity();                                      // lane 0: warp summary
    for (int k = 0; k < nseg; ++k) {
        const int s = k % S;
        rtma::bar_wait(rtma::saddr(&bars[s][warp]), (uint32_t)((k / S) & 1));
        const long long g0 = wbeg + (long long)k * SEG;
        const int cnt = (int)min((long long)SEG, wend - g0);
        const In* sl = seg_ptr(s) + lane * L;
        const long long i0 = g0 + (long long)lane * L;
        T f = M::identity();
        if (cnt == SEG) {
#pragma unroll
            for (int q = 0; q < L / 4; ++q) {
                const int4 v = *reinterpret_cast<const int4*>(sl + 4 * q);
                const In* e = reinterpret_cast<const In*>(&v);
                f = M::combine(f, M::leaf(e[0], i0 + 4 * q));
                f = M::combine(f, M::leaf(e[1], i0 + 4 * q + 1));
                f = M::combine(f, M::leaf(e[2], i0 + 4 * q + 2));
                f = M::combine(f, M::leaf(e[3], i0 + 4 * q + 3));
            }
        } else {                                                // last, partial segment
            const int body = cnt & ~3;
            for (int e = lane * L; e < min(cnt, lane * L + L); ++e)
                f = M::combine(f, M::leaf(e < body ? seg_ptr(s)[e] : x[g0 + e], g0 + e));
        }
        __syncwarp();                                           // reconverge before the tree
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {                      // ordered warp tree
            const T r = reduce_shfl_down(f, o);
            f = M::combine(f, r);   // branch-free (no divergent shuffles)
        }
        if (lane == 0) acc = M::combine(acc, f);
        __syncwarp();
        if (lane == 0 && k + S < nseg) {
            rtma::fence_async();
            issue(k + S);
        }
    }
    if (lane == 0) red[warp] = acc;
    __syncthreads();
    if (tid == 0) {
        T c = M::identity();
        for (int w = 0; w < NW; ++w) c = M::combine(c, red[w]);
        parts[blockIdx.x] = c;
        __threadfence();
        am_last = atomicAdd(ticket, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!am_last) return;
    __threadfence();
    const int np = gridDim.x, per = (np + NT - 1) / NT;
    T a = M::identity();
    for (int q = tid * per; q < min(np, tid * per + per); ++q) {
        T v;
        const volatile int* src = reinterpret_cast<const volatile int*>(parts + q);
        int* dst = reinterpret_cast<int*>(&v);
#pragma unroll
        for (int w = 0; w < (int)(sizeof(T) / 4); ++w) dst[w] = src[w];   // L2-coherent
        a = M::combine(a, v);
    }
    a = reduce_block<M, NT>(a, red);
    if (tid == 0) {
        *out = a;
        *ticket = 0u;
    }
}

// The D&C sum monoid (Alg 4): int32 elements, exact int64 sum.
struct SumI64 {
    using In = int32_t;
    using T = long long;
    static __device__ __forceinline__ T identity() { return 0; }
    static __device__ __forceinline__ T leaf(In x, long long) { return (T)x; }
    static __device__ __forceinline__ T combine(const T& l, const T& r) { return l + r; }
};

// Alg 5 literally: one launch per level, m subproblems,
// a[id] <- a[id] + a[id + m] for id < m (with a bound for odd lengths).
// Valid for the sum because + is commutative; kept as the paper's own layout.
__global__ void alg5_sum_level(long long* __restrict__ a, long long len, long long m) {
    const long long id = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (id < m && id + m < len) a[id] = a[id] + a[id + m];
}

}  // namespace dc
