// sort4_check.cu -- standalone check of the two-level pass kernels
// (nk2_select4, nk3_merge4) against a host reference, one stage at a time.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17
//        -I paper_conf_ipps_lopez_ortizss13_b200/csrc tools/sort4_check.cu -o /tmp/sort4_check
// Usage: sort4_check <n> <w> <dist 0..3> [iters] [max_grid]
#include <cuda_runtime.h>
#include <cstdio>
#ifndef DC_SEL4_MAXROUNDS
#define DC_SEL4_MAXROUNDS 100
#endif

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <random>
#include <vector>

#include "sort_kernels.cuh"
#include "sort4_kernels.cuh"

#define CK(x)                                                                          \
    do {                                                                               \
        cudaError_t e = (x);                                                           \
        if (e != cudaSuccess) {                                                        \
            printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); \
            exit(2);                                                                   \
        }                                                                              \
    } while (0)

#ifndef NT_
#define NT_ 768
#endif
#ifndef IT_
#define IT_ 33
#endif
constexpr int NT = NT_, IT = IT_, T = NT * IT;

int main(int argc, char** argv) {
    setvbuf(stdout, nullptr, _IONBF, 0);
    long long n = argc > 1 ? atoll(argv[1]) : (1 << 22);
    long long w = argc > 2 ? atoll(argv[2]) : 26112;
    int dist = argc > 3 ? atoi(argv[3]) : 0;
    int iters = argc > 4 ? atoi(argv[4]) : 0;
    const int max_grid = argc > 5 ? atoi(argv[5]) : 0;   // >0: few CTAs, many tiles each
    std::mt19937_64 rng(7);
    std::vector<uint32_t> h(n);
    for (long long i = 0; i < n; ++i) {
        uint64_t z = rng();
        h[i] = dist == 0 ? (uint32_t)(z >> 32) : dist == 1 ? (uint32_t)(z & 15)
             : dist == 2 ? 7u : (uint32_t)i;
    }
    for (long long s = 0; s < n; s += w) std::sort(h.begin() + s, h.begin() + std::min(n, s + w));
    const int tpg = (int)((std::min(4 * w, n) + T - 1) / T);
    const int tiles = (int)((n + 4 * w - 1) / (4 * w)) * tpg;
    // host cuts: stable 4-way selection by brute force per group
    std::vector<dc::Cut4> hc(tiles);
    for (auto& c : hc) c.c[0] = c.c[1] = c.c[2] = c.c[3] = -1;   // empty tiles keep -1
    for (long long G = 0; G * 4 * w < n; ++G) {
        long long s = G * 4 * w, l[4];
        for (int q = 0; q < 4; ++q) l[q] = std::max(0LL, std::min(w, n - s - q * w));
        long long tot = l[0] + l[1] + l[2] + l[3];
        long long c[4] = {0, 0, 0, 0};
        long long d = 0;
        for (;;) {
            if (d % T == 0 && d < tot) {
                for (int q = 0; q < 4; ++q) hc[G * tpg + d / T].c[q] = (int)c[q];
            }
            if (d == tot) break;
            int best = -1;
            for (int q = 0; q < 4; ++q) {
                if (c[q] == l[q]) continue;
                if (best < 0 || h[s + q * w + c[q]] < h[s + best * w + c[best]]) best = q;
            }
            c[best]++;
            d++;
        }
    }
    uint32_t *dsrc, *ddst;
    dc::Cut4* dcut;
    CK(cudaMalloc(&dsrc, n * 4));
    CK(cudaMalloc(&ddst, n * 4));
    CK(cudaMalloc(&dcut, (tiles + 1) * sizeof(dc::Cut4)));
    CK(cudaMemcpy(dsrc, h.data(), n * 4, cudaMemcpyHostToDevice));
    CK(cudaMemset(dcut, 0xff, (tiles + 1) * sizeof(dc::Cut4)));
    dc::Pass4 P{};
    for (int q = 0; q < 4; ++q) {
        P.k[q] = dsrc;
        P.v[q] = nullptr;
        P.bound[q] = n;
    }
    P.n = n;
    P.w = w;
    P.T = T;
    P.tpg = tpg;
    P.custom = 0;
    dc::nk2_select4<dc::KeyU32, 2><<<((tiles + dc::sel4_bpw<2>() - 1) / dc::sel4_bpw<2>() + 3) / 4, 128>>>(P, tiles, dcut);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    printf("select4 done\n");
    std::vector<dc::Cut4> gc(tiles);
    CK(cudaMemcpy(gc.data(), dcut, tiles * sizeof(dc::Cut4), cudaMemcpyDeviceToHost));
    int bad = 0;
    for (int j = 0; j < tiles; ++j)
        for (int q = 0; q < 4; ++q)
            if (gc[j].c[q] != hc[j].c[q] && bad++ < 5)
                printf("cut mismatch tile %d run %d: gpu %d host %d\n", j, q, gc[j].c[q], hc[j].c[q]);
    printf("select4: %d mismatches over %d tiles\n", bad, tiles);
    CK(cudaMemcpy(dcut, hc.data(), tiles * sizeof(dc::Cut4), cudaMemcpyHostToDevice));
    auto* k = dc::nk3_merge4<NT, IT, dc::KeyU32, false>;
    const int smem = dc::m4_smem_bytes(T, IT, false);
    CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    int occ = 0, sms = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, NT + 64, smem));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    int grid = std::min(tiles, sms * occ);
    if (max_grid > 0) grid = std::min(grid, max_grid);
    printf("merge4: smem %d B, occupancy %d CTAs/SM, grid %d\n", smem, occ, grid);
    k<<<grid, NT + 64, smem>>>(P, ddst, nullptr, dcut, tiles);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    std::vector<uint32_t> out(n), ref(h);
    CK(cudaMemcpy(out.data(), ddst, n * 4, cudaMemcpyDeviceToHost));
    for (long long s = 0; s < n; s += 4 * w) std::sort(ref.begin() + s, ref.begin() + std::min(n, s + 4 * w));
    long long mism = 0;
    for (long long i = 0; i < n; ++i)
        if (out[i] != ref[i] && mism++ < 5) printf("out mismatch at %lld: %u vs %u\n", i, out[i], ref[i]);
    printf("merge4: %lld mismatches\n", mism);
    if (iters > 0) {
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        float ms_s = 0, ms_m = 0, t;
        for (int i = 0; i < iters; ++i) {
            cudaEventRecord(e0);
            dc::nk2_select4<dc::KeyU32, 2><<<((tiles + dc::sel4_bpw<2>() - 1) / dc::sel4_bpw<2>() + 3) / 4, 128>>>(P, tiles, dcut);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&t, e0, e1);
            if (i) ms_s += t;
            cudaEventRecord(e0);
            k<<<grid, NT + 64, smem>>>(P, ddst, nullptr, dcut, tiles);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            cudaEventElapsedTime(&t, e0, e1);
            if (i) ms_m += t;
        }
        ms_s /= (iters - 1);
        ms_m /= (iters - 1);
        printf("timing: select4 %.4f ms, merge4 %.4f ms (%.1f GB/s)\n", ms_s, ms_m,
               8.0 * n / (ms_m * 1e6));
    }
    return (bad || mism) ? 1 : 0;
}
