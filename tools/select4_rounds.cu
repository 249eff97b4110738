// select4_rounds.cu -- how many rounds does nk2_select4 take per tile boundary?
// n = 2^28 keys as sorted runs of width w (uniform random keys, generated
// sorted on the device: run element i lies in bucket i of 2^32 / w), the
// two-level pass's groups of four runs, tile boundaries every T = 25984
// outputs -- exactly the selection of one pass of the 2^28 sort at run width
// w; prints the rounds histogram and the kernel time for PV = 2 (the keys-only
// default) and PV = 4.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_ipps_lopez_ortizss13_b200/csrc
//      tools/select4_rounds.cu -o /tmp/sel4r
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>
__device__ int g_rounds[1 << 22];
#define DC_SEL4_ROUNDS_OUT g_rounds
#include "sort_kernels.cuh"
#include "sort4_kernels.cuh"

__global__ void gen(uint32_t* k, long long w, long long n, unsigned seed) {
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const long long j = i % w;
    unsigned long long z = (unsigned long long)i * 0x9E3779B97F4A7C15ull + seed;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    z ^= z >> 31;
    const unsigned long long bucket = (1ull << 32) / (unsigned long long)w;
    k[i] = (uint32_t)(j * bucket + (bucket > 1 ? z % bucket : 0));
}

template <int PV>
void run(uint32_t* d, long long n, long long w, int T) {
    dc::Pass4 P{};
    for (int q = 0; q < 4; ++q) { P.k[q] = d; P.v[q] = nullptr; P.bound[q] = n; }
    P.n = n; P.w = w; P.T = T; P.tpg = (int)((std::min(4 * w, n) + T - 1) / T); P.custom = 0;
    const int tiles = (int)(((n + 4 * w - 1) / (4 * w)) * P.tpg);
    dc::Cut4* cuts;
    cudaMalloc(&cuts, sizeof(dc::Cut4) * tiles);
    constexpr int bpw = dc::sel4_bpw<PV>();
    const int warps = (tiles + bpw - 1) / bpw;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    dc::nk2_select4<dc::KeyU32, PV><<<(warps + 3) / 4, 128>>>(P, tiles, cuts);
    cudaEventRecord(a);
    dc::nk2_select4<dc::KeyU32, PV><<<(warps + 3) / 4, 128>>>(P, tiles, cuts);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    std::vector<int> r(tiles);
    cudaMemcpyFromSymbol(r.data(), g_rounds, sizeof(int) * tiles);
    int hist[128] = {0}, mx = 0;
    double avg = 0;
    for (int x : r) { hist[x < 127 ? x : 127]++; mx = x > mx ? x : mx; avg += x; }
    printf("w=%lld PV=%d: %d boundaries, %.1f us, rounds avg %.1f max %d |", w, PV,
           tiles, ms * 1e3, avg / tiles, mx);
    for (int i = 0; i <= mx && i < 128; ++i) if (hist[i]) printf(" %d:%d", i, hist[i]);
    printf("  %s\n", cudaGetErrorString(cudaGetLastError()));
    cudaFree(cuts);
}

int main() {
    const long long n = 1ll << 28;
    uint32_t* d;
    cudaMalloc(&d, n * 4);
    for (long long w = 25088; w < n; w *= 4) {
        // runs of width w over [0, n): element i of run r = key of bucket (i mod w)
        gen<<<(unsigned)((n + 255) / 256), 256>>>(d, w, n, 12345u);
        run<2>(d, n, w, 25984);
        run<4>(d, n, w, 25984);
    }
    cudaFree(d);
    return 0;
}
