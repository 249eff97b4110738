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
template <class M, int NT>
__device__ __forceinline__ typename M::T reduce_block(typename M::T t, typename M::T* red) {
    using T = typename M::T;
    static_assert(NT % 32 == 0 && NT <= 1024, "block of whole warps");
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const T r = reduce_shfl_down(t, off);
        if ((lane & (2 * off - 1)) == 0) t = M::combine(t, r);
    }
    if (lane == 0) red[warp] = t;
    __syncthreads();
    if (warp == 0) {
        t = lane < NT / 32 ? red[lane] : M::identity();
#pragma unroll
        for (int off = 1; off < NT / 32; off <<= 1) {
            const T r = reduce_shfl_down(t, off);
            if ((lane & (2 * off - 1)) == 0) t = M::combine(t, r);
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
