// lds_width_probe.cu -- shared-memory throughput of random per-lane loads of
// different widths, the access pattern of a serial merge-path step (every lane
// reads the next element of its own stream at a data-dependent address).
// Reports elements delivered per SM per cycle and the implied wavefronts per
// warp instruction (1 wavefront = 1 shared-memory cycle per SM).
//   w32      : all lanes, LDS.32 at random word addresses
//   w64      : all lanes, LDS.64 at random 8-byte-aligned addresses
//   w64 half : LDS.64, a random half of the lanes active (predicated)
//   w128     : all lanes, LDS.128 at random 16-byte-aligned addresses
//   w128 q   : LDS.128, a random quarter of the lanes active
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/lds_width_probe.cu -o /tmp/lds_probe
#include <cuda_runtime.h>

#include <cstdio>

constexpr int kIters = 2048;
constexpr int kWords = 8192;    // 32 KB region

__device__ __forceinline__ unsigned hash(unsigned x) {
    x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
    return x;
}

// W = words per load (1, 2, 4); ACT = active-lane fraction numerator over 4
template <int W, int ACT>
__global__ void probe(unsigned* out, long long* cycles) {
    __shared__ __align__(16) unsigned s[kWords];
    for (int i = threadIdx.x; i < kWords; i += blockDim.x) s[i] = hash(i);
    __syncthreads();
    const unsigned base = (unsigned)__cvta_generic_to_shared(s);
    unsigned acc = 0, st = hash(threadIdx.x + 7919u * blockIdx.x);
    const long long t0 = clock64();
#pragma unroll 8
    for (int i = 0; i < kIters; ++i) {
        st = st * 1664525u + 1013904223u;
        const unsigned h = st >> 8;
        const unsigned addr = base + 4u * ((h * W) & (kWords - 1));
        const bool act = ACT == 4 || ((h >> 20) & 3u) < (unsigned)ACT;
        if (W == 1) {
            unsigned v = 0;
            if (act) asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
            acc += v;
        } else if (W == 2) {
            unsigned a = 0, b = 0;
            if (act) asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(a), "=r"(b) : "r"(addr));
            acc += a ^ b;
        } else {
            unsigned a = 0, b = 0, c = 0, d = 0;
            if (act)
                asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];"
                             : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "r"(addr));
            acc += a ^ b ^ c ^ d;
        }
    }
    const long long t1 = clock64();
    if (acc == 0x12345678u) out[0] = acc;
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
}

template <int W, int ACT>
void run(const char* name, unsigned* d_out, long long* d_cyc, int sms) {
    const int threads = 1024;
    probe<W, ACT><<<sms, threads>>>(d_out, d_cyc);
    cudaDeviceSynchronize();
    probe<W, ACT><<<sms, threads>>>(d_out, d_cyc);
    cudaDeviceSynchronize();
    long long h[1024];
    cudaMemcpy(h, d_cyc, sizeof(long long) * sms, cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < sms; ++i) avg += (double)h[i];
    avg /= sms;
    const double warp_instr = (double)(threads / 32) * kIters;     // per SM
    const double elems = warp_instr * 32.0 * W * ACT / 4.0;
    printf("%-10s %7.2f elements/clk/SM  %5.2f clk per warp instruction (= wavefronts when smem-bound)\n",
           name, elems / avg, avg / warp_instr);
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned* d_out;
    long long* d_cyc;
    cudaMalloc(&d_out, 4);
    cudaMalloc(&d_cyc, sizeof(long long) * 1024);
    run<1, 4>("w32", d_out, d_cyc, sms);
    run<1, 2>("w32 half", d_out, d_cyc, sms);
    run<2, 4>("w64", d_out, d_cyc, sms);
    run<2, 2>("w64 half", d_out, d_cyc, sms);
    run<4, 4>("w128", d_out, d_cyc, sms);
    run<4, 1>("w128 q", d_out, d_cyc, sms);
    run<4, 2>("w128 half", d_out, d_cyc, sms);
    return 0;
}
