// Test-only user code of the generic O(1)-combine template include/dc_reduce.cuh
// (SURVEY f4): two NON-commutative user monoids, compiled on the GPU box by
// tests/test_gpu_generic.py and checked against the CPU oracle / Python.
#include <cstdint>

#include "dc_reduce.cuh"

// Max-subarray as a user monoid (combine rules of DESIGN.md Sec. 4).
struct Ms {
    long long tot, pre, suf, best, pe, ss, bs, be;
};
struct MaxsubMonoid {
    using In = int32_t;
    using T = Ms;
    static constexpr long long NEG = -(1LL << 62);
    static __device__ T identity() { return T{0, NEG, NEG, NEG, 0, 0, 0, 0}; }
    static __device__ T leaf(In x, long long i) { return T{x, x, x, x, i, i, i, i}; }
    static __device__ T combine(const T& L, const T& R) {
        T c;
        c.tot = L.tot + R.tot;
        if (L.pre >= L.tot + R.pre) { c.pre = L.pre; c.pe = L.pe; }
        else { c.pre = L.tot + R.pre; c.pe = R.pe; }
        if (R.tot + L.suf >= R.suf) { c.suf = R.tot + L.suf; c.ss = L.ss; }
        else { c.suf = R.suf; c.ss = R.ss; }
        c.best = L.best; c.bs = L.bs; c.be = L.be;
        if (L.suf + R.pre > c.best) { c.best = L.suf + R.pre; c.bs = L.ss; c.be = R.pe; }
        if (R.best > c.best) { c.best = R.best; c.bs = R.bs; c.be = R.be; }
        return c;
    }
};

// Polynomial hash sum_i x_i * B^(len-1-i) mod 2^64: order-sensitive.
struct Hash {
    unsigned long long h, p;   // hash, B^len
};
struct HashMonoid {
    using In = int32_t;
    using T = Hash;
    static constexpr unsigned long long B = 1000003ULL;
    static __device__ T identity() { return T{0ULL, 1ULL}; }
    static __device__ T leaf(In x, long long) { return T{(unsigned long long)(unsigned)x, B}; }
    static __device__ T combine(const T& l, const T& r) { return T{l.h * r.p + r.h, l.p * r.p}; }
};

template <class M>
static int run(const int32_t* x, long long n, void* parts, void* ticket, void* out) {
    constexpr int NT = 128, C = 16;
    const long long tiles = (n + NT * C - 1) / (NT * C);
    const int grid = (int)(tiles < 300 ? tiles : 300);
    dc::breadth_first_reduce<M, NT, C><<<grid, NT>>>(x, n, (typename M::T*)parts,
                                                     (unsigned int*)ticket, (typename M::T*)out);
    return (int)cudaDeviceSynchronize();
}

// The TMA-streamed variant (warp segments of 32 x 36 elements, 3 stages).
template <class M>
static int run_tma(const int32_t* x, long long n, void* parts, void* ticket, void* out) {
    constexpr int NT = 128, L = 36, S = 3;
    constexpr size_t smem = dc::breadth_first_reduce_tma_smem<NT, L, S>();
    auto* k = dc::breadth_first_reduce_tma<M, NT, L, S>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const long long units = (n + NT * L - 1) / (NT * L);
    const int grid = (int)(units < 300 ? (units > 0 ? units : 1) : 300);
    k<<<grid, NT, smem>>>(x, n, dc::breadth_first_reduce_tma_rw<NT, L>(n, grid),
                          (typename M::T*)parts, (unsigned int*)ticket, (typename M::T*)out);
    return (int)cudaDeviceSynchronize();
}

extern "C" int demo_maxsub_tma(const int32_t* x, long long n, void* parts, void* ticket,
                               void* out) {
    return run_tma<MaxsubMonoid>(x, n, parts, ticket, out);
}
extern "C" int demo_hash_tma(const int32_t* x, long long n, void* parts, void* ticket, void* out) {
    return run_tma<HashMonoid>(x, n, parts, ticket, out);
}

extern "C" int demo_maxsub(const int32_t* x, long long n, void* parts, void* ticket, void* out) {
    return run<MaxsubMonoid>(x, n, parts, ticket, out);
}
extern "C" int demo_hash(const int32_t* x, long long n, void* parts, void* ticket, void* out) {
    return run<HashMonoid>(x, n, parts, ticket, out);
}
