// stream_probe.cu -- how fast can one kernel stream a 64 MB int32 array out
// of HBM (L2 flushed by a 512 MiB read before every launch)?  The max-subarray
// NK4 and the D&C sum read their input once, so this is their floor.  Every
// variant computes an int64 sum (checked) so the loads cannot be elided.
//   ldg     : grid-stride coalesced 128-bit loads, CTAS x 256 threads, U-unrolled
//   tma_w   : per-warp 1-D TMA bulk segments of 32*L words, S-stage ring (NK4's scheme)
//   tma_c   : per-CTA TMA bulk chunks of C bytes, S-stage ring, all warps consume
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/stream_probe.cu -o /tmp/stream_probe
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t ph) {
    uint32_t done;
    do {
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(done) : "r"(bar), "r"(ph) : "memory");
    } while (!done);
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}

__device__ unsigned long long g_sum;

__device__ __forceinline__ void block_add(long long v) {
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0) atomicAdd(&g_sum, (unsigned long long)v);
}

template <int U>
__global__ void __launch_bounds__(256) k_ldg(const int4* __restrict__ x, long long n4) {
    long long s = 0;
    const long long stride = (long long)gridDim.x * 256;
    long long i = (long long)blockIdx.x * 256 + threadIdx.x;
    for (; i + (U - 1) * stride < n4; i += U * stride) {
        int4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = __ldcs(x + i + u * stride);
#pragma unroll
        for (int u = 0; u < U; ++u) s += (long long)v[u].x + v[u].y + v[u].z + v[u].w;
    }
    for (; i < n4; i += stride) { int4 v = __ldcs(x + i); s += (long long)v.x + v.y + v.z + v.w; }
    block_add(s);
}

// per-warp segments (NK4 scheme): NW warps, S stages of 32*L words per warp
template <int NW, int L, int S>
__global__ void __launch_bounds__(NW * 32, 1) k_tma_w(const int* __restrict__ x, long long n, long long RW) {
    constexpr int SEG = 32 * L;
    extern __shared__ __align__(16) int sm[];
    __shared__ __align__(8) uint64_t bars[S][NW];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const long long wbeg = min(n, ((long long)blockIdx.x * NW + warp) * RW);
    const long long wend = min(n, wbeg + RW);
    const int nseg = (int)((wend - wbeg) / SEG);    // probe sizes are whole segments
    if (lane == 0) for (int s = 0; s < S; ++s) mbar_init(smem_addr(&bars[s][warp]), 1);
    __syncwarp();
    auto buf = [&](int s) { return sm + (s * NW + warp) * SEG; };
    auto issue = [&](int k) {
        const int s = k % S;
        const uint32_t b = smem_addr(&bars[s][warp]);
        mbar_expect(b, 4u * SEG);
        bulk_g2s(smem_addr(buf(s)), x + wbeg + (long long)k * SEG, 4u * SEG, b);
    };
    if (lane == 0) for (int k = 0; k < S && k < nseg; ++k) issue(k);
    long long acc = 0;
    for (int k = 0; k < nseg; ++k) {
        const int s = k % S;
        mbar_wait(smem_addr(&bars[s][warp]), (k / S) & 1);
        const int* p = buf(s) + lane * L;
#pragma unroll
        for (int q = 0; q < L; q += 4) {
            const int4 v = *reinterpret_cast<const int4*>(p + q);
            acc += (long long)v.x + v.y + v.z + v.w;
        }
        __syncwarp();
        if (lane == 0 && k + S < nseg) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            issue(k + S);
        }
    }
    block_add(acc);
}

// per-CTA chunks: thread 0 issues C-byte bulk copies into an S-stage ring;
// full[s] (TMA bytes), empty[s] (one arrive per warp)
template <int NT, int C, int S>
__global__ void __launch_bounds__(NT, 1) k_tma_c(const int* __restrict__ x, long long n) {
    constexpr int W = C / 4;
    extern __shared__ __align__(16) int sm[];
    __shared__ __align__(8) uint64_t full[S], empty[S];
    const long long nchunk = n / W;
    const long long my = (nchunk - blockIdx.x + gridDim.x - 1) / gridDim.x;   // chunks b, b+G, ...
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(smem_addr(&full[s]), 1); mbar_init(smem_addr(&empty[s]), NT / 32); }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int k = 0; k < S && k < my; ++k) {
            mbar_expect(smem_addr(&full[k]), C);
            bulk_g2s(smem_addr(sm + k * W), x + (blockIdx.x + (long long)k * gridDim.x) * W, C, smem_addr(&full[k]));
        }
    }
    long long acc = 0;
    for (long long k = 0; k < my; ++k) {
        const int s = (int)(k % S);
        const uint32_t ph = (uint32_t)((k / S) & 1);
        mbar_wait(smem_addr(&full[s]), ph);
        const int4* p = reinterpret_cast<const int4*>(sm + s * W);
        for (int q = threadIdx.x; q < W / 4; q += NT) {
            const int4 v = p[q];
            acc += (long long)v.x + v.y + v.z + v.w;
        }
        __syncwarp();
        if ((threadIdx.x & 31) == 0) mbar_arrive(smem_addr(&empty[s]));
        if (threadIdx.x == 0 && k + S < my) {
            mbar_wait(smem_addr(&empty[s]), ph);
            mbar_expect(smem_addr(&full[s]), C);
            bulk_g2s(smem_addr(sm + s * W), x + (blockIdx.x + (k + S) * gridDim.x) * W, C, smem_addr(&full[s]));
        }
    }
    block_add(acc);
}

__global__ void k_flush(const int4* __restrict__ f, long long n4, int* sink) {
    int s = 0;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (long long)gridDim.x * blockDim.x) {
        const int4 v = __ldcs(f + i);
        s ^= v.x ^ v.w;
    }
    if (s == 0x7fffffff) *sink = s;
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const long long flush_bytes = 512ll << 20;
    int4* flush;
    int* sink;
    CK(cudaMalloc(&flush, flush_bytes));
    CK(cudaMemset(flush, 1, flush_bytes));
    CK(cudaMalloc(&sink, 4));
    for (long long n : {1ll << 24, 1ll << 26}) {
        int* x;
        CK(cudaMalloc(&x, n * 4));
        std::vector<int> h(n);
        long long ref = 0;
        for (long long i = 0; i < n; ++i) { h[i] = (int)((i * 2654435761ll) % 2001) - 1000; ref += h[i]; }
        CK(cudaMemcpy(x, h.data(), n * 4, cudaMemcpyHostToDevice));
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        auto timeit = [&](const char* name, auto launch) {
            float best = 1e9, sum = 0;
            const int reps = 20;
            bool ok = true;
            for (int r = 0; r < reps + 2; ++r) {
                k_flush<<<sms * 4, 512>>>(flush, flush_bytes / 16, sink);
                unsigned long long z = 0;
                cudaMemcpyToSymbol(g_sum, &z, 8);
                cudaEventRecord(e0);
                launch();
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                float ms;
                cudaEventElapsedTime(&ms, e0, e1);
                unsigned long long got;
                cudaMemcpyFromSymbol(&got, g_sum, 8);
                if ((long long)got != ref) ok = false;
                if (r >= 2) { best = ms < best ? ms : best; sum += ms; }
            }
            const cudaError_t err = cudaGetLastError();
            printf("n=2^%d %-26s best %7.2f us  avg %7.2f us  %6.0f GB/s (avg)  %s%s\n", n == (1ll << 24) ? 24 : 26, name,
                   best * 1e3, sum / reps * 1e3, n * 4 / (sum / reps * 1e-3) / 1e9, ok ? "ok" : "WRONG",
                   err == cudaSuccess ? "" : cudaGetErrorString(err));
        };
        for (int cpsm : {2, 4, 8, 16}) {
            char nm[64];
            snprintf(nm, sizeof nm, "ldg U=4 %d CTA/SM", cpsm);
            timeit(nm, [&] { k_ldg<4><<<sms * cpsm, 256>>>((const int4*)x, n / 4); });
        }
        timeit("ldg U=8 8 CTA/SM", [&] { k_ldg<8><<<sms * 8, 256>>>((const int4*)x, n / 4); });
        {
            // NK4's scheme: 8 warps, L=68, S=2; RW = per-warp range (whole segments)
            constexpr int NW = 8, L = 68, S = 2, SEG = 32 * L;
            const long long warps = (long long)sms * NW;
            long long RW = (n + warps - 1) / warps;
            RW = (RW + SEG - 1) / SEG * SEG;
            const int smem = S * NW * SEG * 4;
            cudaFuncSetAttribute(k_tma_w<NW, L, S>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            const int grid = (int)((n + NW * RW - 1) / (NW * RW));
            timeit("tma_w NW8 L68 S2", [&] { k_tma_w<NW, L, S><<<grid, NW * 32, smem>>>(x, n, RW); });
        }
        {
            constexpr int NW = 16, L = 36, S = 3, SEG = 32 * L;
            const long long warps = (long long)sms * NW;
            long long RW = (n + warps - 1) / warps;
            RW = (RW + SEG - 1) / SEG * SEG;
            const int smem = S * NW * SEG * 4;
            cudaFuncSetAttribute(k_tma_w<NW, L, S>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            const int grid = (int)((n + NW * RW - 1) / (NW * RW));
            timeit("tma_w NW16 L36 S3", [&] { k_tma_w<NW, L, S><<<grid, NW * 32, smem>>>(x, n, RW); });
        }
        {
            constexpr int NT = 512, C = 16384, S = 12;
            cudaFuncSetAttribute(k_tma_c<NT, C, S>, cudaFuncAttributeMaxDynamicSharedMemorySize, C * S);
            timeit("tma_c 16KB x12 512t", [&] { k_tma_c<NT, C, S><<<sms, NT, C * S>>>(x, n); });
        }
        {
            constexpr int NT = 512, C = 32768, S = 6;
            cudaFuncSetAttribute(k_tma_c<NT, C, S>, cudaFuncAttributeMaxDynamicSharedMemorySize, C * S);
            timeit("tma_c 32KB x6 512t", [&] { k_tma_c<NT, C, S><<<sms, NT, C * S>>>(x, n); });
        }
        {
            constexpr int NT = 256, C = 8192, S = 12;
            cudaFuncSetAttribute(k_tma_c<NT, C, S>, cudaFuncAttributeMaxDynamicSharedMemorySize, C * S);
            timeit("tma_c 8KB x12 256t 2/SM", [&] { k_tma_c<NT, C, S><<<sms * 2, NT, C * S>>>(x, n); });
        }
        cudaFree(x);
    }
    return 0;
}
