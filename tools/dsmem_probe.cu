// dsmem_probe.cu -- B200 measurement for the f2 decision:
// distributed-shared-memory read bandwidth between the CTAs of a cluster vs
// local shared memory, with every SM busy (one cluster-pair CTA per SM).
// Each CTA fills WORDS words of its shared memory, the cluster syncs, then
// every thread reads the PARTNER's (or its own) shared memory with 128-bit
// loads, REPS times.  Prints bytes/cycle/SM.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/dsmem tools/dsmem_probe.cu
#include <cooperative_groups.h>
#include <cstdio>

namespace cg = cooperative_groups;

constexpr int WORDS = 26112;   // one NK1 tile (104 KB)
constexpr int REPS = 8;

template <bool REMOTE>
__global__ void __cluster_dims__(2, 1, 1) probe(unsigned long long* cycles, int* sink) {
    extern __shared__ __align__(16) int sm[];
    cg::cluster_group cl = cg::this_cluster();
    for (int i = threadIdx.x; i < WORDS; i += blockDim.x) sm[i] = i * 7 + blockIdx.x;
    cl.sync();
    const int* src = REMOTE ? cl.map_shared_rank(sm, cl.block_rank() ^ 1) : sm;
    int acc = 0;
    const unsigned long long t0 = clock64();
    for (int r = 0; r < REPS; ++r) {
#pragma unroll 4
        for (int i = 4 * threadIdx.x; i < WORDS; i += 4 * blockDim.x) {
            const int4 v = *reinterpret_cast<const int4*>(src + ((i + r * 64) % WORDS));
            acc += v.x ^ v.y ^ v.z ^ v.w;
        }
    }
    __syncthreads();
    const unsigned long long t1 = clock64();
    cl.sync();
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
    if (acc == 0x12345) sink[0] = acc;
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int grid = sms - (sms & 1);
    const size_t smem = WORDS * 4;
    unsigned long long* cyc;
    int* sink;
    cudaMalloc(&cyc, grid * 8);
    cudaMalloc(&sink, 4);
    cudaFuncSetAttribute(probe<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(probe<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    for (int remote = 0; remote < 2; ++remote) {
        for (int it = 0; it < 3; ++it) {
            if (remote) probe<true><<<grid, 512, smem>>>(cyc, sink);
            else probe<false><<<grid, 512, smem>>>(cyc, sink);
        }
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
        unsigned long long* h = new unsigned long long[grid];
        cudaMemcpy(h, cyc, grid * 8, cudaMemcpyDeviceToHost);
        double mean = 0;
        for (int b = 0; b < grid; ++b) mean += h[b];
        mean /= grid;
        const double bytes = (double)WORDS * 4 * REPS;
        printf("%s smem reads: %.1f B/cycle/SM (%d CTAs, %.0f cycles for %.0f KB)\n",
               remote ? "DSMEM (partner CTA)" : "local", bytes / mean, grid, mean, bytes / 1024);
        delete[] h;
    }
    return 0;
}
