// mio_probe.cu -- B200 throughput of the MIO-side operations a merge level is
// built from: __shfl_xor_sync, conflict-free LDS, and LDS at random per-lane
// addresses (the serial merge-path pattern).  One number per op: warp
// instructions per SM per cycle (1.0 = one 32-lane op per clock per SM).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/mio_probe.cu -o /tmp/mio_probe
#include <cuda_runtime.h>

#include <cstdio>

constexpr int kIters = 4096;

__global__ void shfl_kernel(unsigned* out) {
    unsigned v = threadIdx.x * 2654435761u, acc = 0;
#pragma unroll 16
    for (int i = 0; i < kIters; ++i) {
        v = __shfl_xor_sync(0xffffffffu, v, (i & 15) + 1) + i;
        acc ^= v;
    }
    if (acc == 0x12345678u) out[0] = acc;
}

template <bool RANDOM>
__global__ void lds_kernel(unsigned* out) {
    __shared__ unsigned s[8192];
    for (int i = threadIdx.x; i < 8192; i += blockDim.x) s[i] = i * 2654435761u;
    __syncthreads();
    unsigned idx = RANDOM ? (threadIdx.x * 2654435761u) & 8191 : threadIdx.x, acc = 0;
#pragma unroll 16
    for (int i = 0; i < kIters; ++i) {
        const unsigned v = s[idx];
        acc += v;
        // random: next index from the loaded value (data-dependent, like a merge);
        // conflict-free: lane-consecutive words
        idx = RANDOM ? ((idx + (v & 63) + 1) & 8191) : ((idx + 32) & 8191);
    }
    if (acc == 0x12345678u) out[0] = acc;
}

int main() {
    unsigned* d;
    cudaMalloc(&d, 4);
    int sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);   // kHz
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int blocks = sms * 8, threads = 256;
    auto run = [&](const char* name, auto launch) {
        launch();
        cudaEventRecord(a);
        for (int r = 0; r < 5; ++r) launch();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        const double warp_ops = 5.0 * blocks * (threads / 32) * (double)kIters;
        const double cycles = ms * 1e-3 * clk * 1e3;
        printf("%-22s %.3f warp-ops / SM / cycle  (%.3f ms, %d SMs, %.0f MHz nominal)\n", name,
               warp_ops / sms / cycles, ms / 5, sms, clk / 1e3);
    };
    run("shfl_xor", [&] { shfl_kernel<<<blocks, threads>>>(d); });
    run("lds conflict-free", [&] { lds_kernel<false><<<blocks, threads>>>(d); });
    run("lds random lanes", [&] { lds_kernel<true><<<blocks, threads>>>(d); });
    cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
