// nk4_trace.cu -- timeline of one NK4 launch (max-subarray, 2^24 int32) from
// %globaltimer stamps the kernel writes when built with -DDC_MS_TRACE: CTA
// entry, end of every warp's segment loop, CTA ticket, end of the last CTA.
// L2 flushed by a 512 MiB read before the launch, like bench.py.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -DDC_MS_TRACE -I include
//      -I paper_conf_ipps_lopez_ortizss13_b200/csrc tools/nk4_trace.cu -o /tmp/nk4_trace
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>

#include "dc.h"
namespace dc { __device__ unsigned long long dc_ms_trace[2048 * 16 + 16]; }
#include "maxsub_tma.cuh"
using dc::dc_ms_trace;

__global__ void flush_read(const int4* f, long long n4, int* sink) {
    extern __shared__ int dyn[];   // (the variant launch asks for NK4's carveout)
    if (n4 < 0) dyn[threadIdx.x] = 0;
    int s = 0;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (long long)gridDim.x * blockDim.x) {
        const int4 v = __ldcs(f + i);
        s ^= v.x;
    }
    if (s == 0x7fffffff) *sink = s;
}

__global__ void empty_kernel(int* sink) {
    extern __shared__ int dyn[];
    if (sink == nullptr) dyn[threadIdx.x] = 0;
}

int main(int argc, char** argv) {
    constexpr int NT = 256, L = 76, S = 2, J = 2;   // the library default
    const long long n = 1ll << 24;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    std::vector<int> h(n);
    unsigned long long z = 88172645463325252ull;
    for (auto& v : h) { z ^= z << 13; z ^= z >> 7; z ^= z << 17; v = (int)(z >> 32); }
    int *x, *sink;
    int4* fl;
    dc_maxsub_tuple* parts;
    unsigned* ticket;
    dc_maxsub_result* res;
    cudaMalloc(&x, n * 4);
    cudaMemcpy(x, h.data(), n * 4, cudaMemcpyHostToDevice);
    cudaMalloc(&fl, 512ll << 20);
    cudaMemset(fl, 1, 512ll << 20);
    cudaMalloc(&sink, 4);
    cudaMalloc(&parts, 4096 * sizeof(dc_maxsub_tuple));
    cudaMalloc(&ticket, 4);
    cudaMemset(ticket, 0, 4);
    cudaMalloc(&res, sizeof(dc_maxsub_result));
#ifndef DC_MS_VONLY
#define DC_MS_VONLY 1
#endif
    auto k = dc::nk4_maxsub_tma<NT, L, S, J, DC_MS_VONLY != 0>;
    const int smem = S * NT * L * 4;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const long long warps = (long long)sms * (NT / 32), seg = 32ll * L;
    const long long R = ((n + warps - 1) / warps + seg - 1) / seg * seg;
    const int grid = sms;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaFuncSetAttribute(flush_read, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (int rep = 0; rep < 8; ++rep) {
        // reps 0-3: the flush kernel uses no shared memory (like bench.py's torch
        // read); reps 4-7: it reserves NK4's dynamic shared memory, so the SMs
        // keep the same L1/shared carveout across the two launches
        if (rep < 4) flush_read<<<sms * 4, 512>>>(fl, (512ll << 20) / 16, sink);
        else flush_read<<<sms, 512, smem>>>(fl, (512ll << 20) / 16, sink);
        cudaMemset(dc_ms_trace, 0, 0);  // no-op; keep symbol referenced
        cudaEventRecord(e0);
        k<<<grid, NT, smem>>>(x, n, R, parts, ticket, 0, 0, res, nullptr);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        std::vector<unsigned long long> t(2048 * 16 + 16);
        cudaMemcpyFromSymbol(t.data(), dc_ms_trace, t.size() * 8);
        unsigned long long t0 = ~0ull, start_max = 0, loop_end_max = 0, tick_max = 0;
        std::vector<double> loop_end, start;
        const int active = (int)std::min<long long>(grid, (n + (NT / 32) * R - 1) / ((NT / 32) * R));
        for (int b = 0; b < active; ++b) t0 = std::min(t0, t[b * 16]);
        for (int b = 0; b < active; ++b) {
            start.push_back((t[b * 16] - t0) / 1e3);
            start_max = std::max(start_max, t[b * 16] - t0);
            for (int w = 0; w < NT / 32; ++w) {
                loop_end.push_back((t[b * 16 + 1 + w] - t0) / 1e3);
                loop_end_max = std::max(loop_end_max, t[b * 16 + 1 + w] - t0);
            }
            tick_max = std::max(tick_max, t[b * 16 + 15] - t0);
        }
        std::sort(loop_end.begin(), loop_end.end());
        std::sort(start.begin(), start.end());
        const double last = (t[2047 * 16] - t0) / 1e3;
        printf("rep %d: event %.2f us | CTAs %d, R=%lld | start: median %.2f max %.2f us | warp loop end: min %.2f median %.2f p90 %.2f max %.2f us | last ticket %.2f us | last CTA done %.2f us\n",
               rep, ms * 1e3, active, R, start[start.size() / 2], start_max / 1e3, loop_end.front(),
               loop_end[loop_end.size() / 2], loop_end[loop_end.size() * 9 / 10], loop_end_max / 1e3,
               tick_max / 1e3, last);
    }
    // launch floor: an empty kernel of the same grid, block and shared memory
    cudaFuncSetAttribute(empty_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (int rep = 0; rep < 3; ++rep) {
        flush_read<<<sms * 4, 512>>>(fl, (512ll << 20) / 16, sink);
        cudaEventRecord(e0);
        empty_kernel<<<grid, NT, smem>>>(sink);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        cudaEventRecord(e0);
        empty_kernel<<<grid, NT, smem>>>(sink);
        empty_kernel<<<grid, NT, smem>>>(sink);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms2;
        cudaEventElapsedTime(&ms2, e0, e1);
        printf("empty kernel (grid %d x %d, %d B smem) after the flush: %.2f us; two back to back: %.2f us\n", grid, NT, smem, ms * 1e3, ms2 * 1e3);
    }
    dc_maxsub_result r;
    cudaMemcpy(&r, res, sizeof r, cudaMemcpyDeviceToHost);
    printf("result sum %lld [%lld, %lld]  (%s)\n", (long long)r.sum, (long long)r.start, (long long)r.end,
           cudaGetErrorString(cudaGetLastError()));
    return 0;
}
