// racecheck_mbar_probe.cu -- does compute-sanitizer racecheck model an mbarrier
// hand-off between a generic-proxy shared store and a later TMA (async-proxy)
// write of the same words?  Warp 0 stores a buffer, fences (proxy.async), and
// arrives on an mbarrier; warp 1 waits on it and then overwrites the buffer by
// a bulk copy.  The order is guaranteed by the release/acquire of the mbarrier
// (the same hand-off nk3_merge4 uses between its consumers and its producer).
// Run: compute-sanitizer --tool racecheck /tmp/racecheck_mbar_probe
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

#include "sort_kernels.cuh"

__global__ void probe(const uint32_t* __restrict__ g, uint32_t* __restrict__ out) {
    __shared__ __align__(16) uint32_t buf[256];
    __shared__ __align__(8) uint64_t empty, full;
    const int tid = threadIdx.x;
    if (tid == 0) {
        dc::mbar_init(dc::smem_addr(&empty), 1);
        dc::mbar_init(dc::smem_addr(&full), 1);
    }
    __syncthreads();
    if (tid < 32) {                                   // "consumer": generic writes, then release
        for (int i = tid; i < 256; i += 32) buf[i] = i;
        dc::fence_proxy_async_smem();
        __syncwarp();
        if (tid == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(dc::smem_addr(&empty)) : "memory");
    } else if (tid < 64) {                            // "producer": acquire, then TMA overwrite
        dc::mbar_wait(dc::smem_addr(&empty), 0);
        if (tid == 32) {
            dc::mbar_arrive_expect_tx(dc::smem_addr(&full), 1024);
            dc::bulk_g2s(dc::smem_addr(buf), g, 1024, dc::smem_addr(&full));
        }
        dc::mbar_wait(dc::smem_addr(&full), 0);
        for (int i = tid - 32; i < 256; i += 32) out[i] = buf[i];
    }
}

int main() {
    uint32_t *g, *o;
    cudaMalloc(&g, 1024);
    cudaMalloc(&o, 1024);
    cudaMemset(g, 7, 1024);
    probe<<<1, 64>>>(g, o);
    uint32_t h[256];
    cudaMemcpy(h, o, 1024, cudaMemcpyDeviceToHost);
    printf("probe %s, out[5] = 0x%08x (expect 0x07070707)\n", cudaGetErrorString(cudaGetLastError()), h[5]);
    return 0;
}
