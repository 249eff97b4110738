// dc_api.cu -- the C ABI (include/dc.h): plans, the level driver and launches.
//
// Layer a0 (plan): the level table of T(n) = aT(n/b) + f(n) (P:L236,
// P:L425-439) and the execution schedule (fused bottom levels + global merge
// passes).  Layer a4 (level driver): Alg 7's recursion unrolled bottom-up
// (Alg 2): NK1 once, then for every remaining level NK2 + NK3 with
// src/dst ping-pong over the paper's 2n working space, the
// parity chosen so that the last pass lands in the caller's buffer.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <algorithm>
#include <atomic>
#include <new>
#include <string>
#include <vector>

#include "dc.h"
#include "plan.h"
#include "dc_reduce.cuh"
#include "maxsub_kernels.cuh"
#include "mg_kernels.cuh"
#include "sort_kernels.cuh"
#include "sort4_kernels.cuh"
#include "maxsub_tma.cuh"
#include "maxsub_rows.cuh"

#include <cudaTypedefs.h>
#include <mutex>

namespace {

// ---------------------------------------------------------------- config
// Sort configuration per instantiation (tuned on B200 with tools/sweep.sh,
// see DESIGN.md Sec. 5).  Keys-only u32/i32 (stability unobservable): NK1 of
// 512 threads x 49 items = tiles of 25088 keys (9 shared-memory merge levels
// on top of a 49-input register network; 14 global levels at 2^28), one-level
// merge CTAs of 256 x 51 = 13056 outputs.  49 rather than 51 items: a group of
// four 25088-key runs splits into four 4-way tiles of <= 25984 keys, where four
// 26112-key runs need a fifth 3072-key sliver tile (2^28: 6.08 -> 5.96 ms).
// (1024 x 51 tiles save a global level at 2^28 but cost more in NK1 than they
// save: 6.38 vs 6.19 ms.)  f32 keys carry a tile-local index for stability:
// 512 x 33 = 16896-key tiles, merge CTAs of 256 x 33 outputs; key-value
// NK1 uses 256-thread CTAs (kCfgKV).  Merge tiles need not divide a pair:
// every pair is cut into ceil(2w / tout) tiles, the last one short.
struct SortCfg {
    int nt1, it1, nt3, it;   // NK1 threads x items, one-level merge threads x items
    constexpr int tile() const { return nt1 * it1; }
    constexpr int tout() const { return nt3 * it; }
};
#ifndef DC_FAST_NT1
#define DC_FAST_NT1 512
#endif
#ifndef DC_FAST_IT1
#define DC_FAST_IT1 49
#endif
#ifndef DC_FAST_IT
#define DC_FAST_IT 51
#endif
#ifndef DC_FAST_NT3
#define DC_FAST_NT3 256
#endif
#ifndef DC_STABLE_NT1
#define DC_STABLE_NT1 512
#endif
#ifndef DC_STABLE_IT
#define DC_STABLE_IT 33
#endif
#ifndef DC_STABLE_NT3
#define DC_STABLE_NT3 256
#endif
constexpr SortCfg kCfgFast{DC_FAST_NT1, DC_FAST_IT1, DC_FAST_NT3, DC_FAST_IT};
constexpr SortCfg kCfgStable{DC_STABLE_NT1, DC_STABLE_IT, DC_STABLE_NT3, DC_STABLE_IT};
// Key-value NK1: (key, index) pairs in registers need ~107 registers, so a
// 512-thread CTA runs alone on its SM (16 warps, latency-bound); 256-thread
// CTAs run two per SM.  Their 8448-key tiles cost one more global level, but
// NK1 drops 4.45 -> 3.33 ms at 2^28 (11.71 -> 11.23 ms per sort, measured).
#ifndef DC_KV_NT1
#define DC_KV_NT1 256
#endif
#ifndef DC_KV_IT1
#define DC_KV_IT1 DC_STABLE_IT
#endif
constexpr SortCfg kCfgKV{DC_KV_NT1, DC_KV_IT1, DC_STABLE_NT3, DC_STABLE_IT};
// Small inputs (n < kSmallN, L2-resident): quarter-size tiles so that the
// fused kernel and every merge level still launch >= ~150 CTAs.
#ifndef DC_SMALL_NT1
#define DC_SMALL_NT1 128
#endif
#ifndef DC_SMALL_IT1   // 128 x 49 = 6272: four quarter runs fill one 4-way tile (25088 <= 25984)
#define DC_SMALL_IT1 49
#endif
constexpr SortCfg kCfgFastSmall{DC_SMALL_NT1, DC_SMALL_IT1, 128, DC_FAST_IT};
constexpr SortCfg kCfgStableSmall{128, DC_STABLE_IT, 128, DC_STABLE_IT};
constexpr int cmin(int a, int b) { return a < b ? a : b; }
constexpr int kMinTout = cmin(cmin(cmin(kCfgFast.tout(), kCfgStable.tout()), kCfgKV.tout()),
                              cmin(kCfgFastSmall.tout(), kCfgStableSmall.tout()));

template <class K, bool V, bool SMALL>
constexpr SortCfg cfg_for() {
    return V ? (SMALL ? kCfgStableSmall : kCfgKV)
           : K::kNeedStable ? (SMALL ? kCfgStableSmall : kCfgStable)
                                 : (SMALL ? kCfgFastSmall : kCfgFast);
}
SortCfg cfg_for_runtime(dc_key_type kt, bool vals, bool small) {
    return vals ? (small ? kCfgStableSmall : kCfgKV)
           : kt == DC_KEY_F32 ? (small ? kCfgStableSmall : kCfgStable)
                                      : (small ? kCfgFastSmall : kCfgFast);
}

#ifndef DC_MS_NT
#define DC_MS_NT 256
#endif
#ifndef DC_MS_C
#define DC_MS_C 256
#endif
constexpr int kNK4Threads = DC_MS_NT;
constexpr int kNK4Chunk = DC_MS_C;
constexpr int kMsTile = kNK4Threads * kNK4Chunk;   // values per max-subarray CTA

constexpr int64_t kMaxN = 2147483647LL;

thread_local std::string g_last_error;

dc_status fail(dc_status s, const std::string& msg) {
    g_last_error = msg;
    return s;
}

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

int nk1_smem_bytes(SortCfg c, bool vals) {
    return (vals ? (DC_NK1_KV_LATE ? 2 : 3) : 1) * dc::tile_words(c.tile(), 0) * 4;
}
int nk3_smem_bytes(SortCfg c, bool vals) {
    return (vals ? 2 : 1) * dc::tile_words(c.tout(), c.it + 16) * 4;
}

}  // namespace


namespace {

int64_t num_tiles(int64_t n, int64_t t) { return (n + t - 1) / t; }

int global_passes(int64_t n, int64_t tile) {
    int p = 0;
    for (int64_t w = tile; w < n; w *= 2) ++p;
    return p;
}

// One-level pass: every pair of width 2w is cut into ceil(2w / tout) tiles, so
// at most one extra (short) tile per pair; pairs <= n / (2 * min tile) + 1.
constexpr int kMinTile = cmin(cmin(cmin(kCfgFast.tile(), kCfgStable.tile()), kCfgKV.tile()),
                              cmin(kCfgFastSmall.tile(), kCfgStableSmall.tile()));
size_t split_entries(int64_t n) {
    return (size_t)num_tiles(n, kMinTout) + (size_t)num_tiles(n, 2 * (int64_t)kMinTile) + 2;
}

// Two-level passes: 4-way output tiles of NT*IT keys, one cut vector (4 ints)
// per tile; every group of 4 runs is cut into ceil(min(4w, n)/T) tiles.  Keys
// only: 896 x 29 (T = 25984; one CTA per SM, 2 x 104 KB of buffers); with
// values the key and value regions share the same budget: 512 x 25.
// r02: 896 x 29 (T = 25984, 960 threads x 64 registers) 3.708 ms of merges per
// 2^28 u32 sort vs 768 x 33 3.757; fewer threads with more items are slower
// (512 x 49 4.03 ... 320 x 79 4.92; profiles/r02/m4_shapes.txt).
#ifndef DC_TWO_NT
#define DC_TWO_NT 896
#endif
#ifndef DC_TWO_IT
#define DC_TWO_IT 29
#endif
#ifndef DC_TWO_NT_KV
#define DC_TWO_NT_KV 512
#endif
#ifndef DC_TWO_IT_KV
#define DC_TWO_IT_KV 25
#endif
// (Selection fused into the pass -- selector warps inside nk3_merge4 -- was
// measured slower at 2^28: merges + selection 5.02 / 4.70 ms with 3 / 6
// selector warps vs 4.36 ms for the separate nk2_select4 launch: a
// boundary's ~11 dependent rounds need many warps in flight, which a separate
// full-GPU launch provides and a few warps per SM do not.  Removed in r02.)
struct TwoCfg {
    int nt, it;
    constexpr int T() const { return nt * it; }
    constexpr int threads() const { return nt + 64; }
};
constexpr TwoCfg kTwoKeys{DC_TWO_NT, DC_TWO_IT};
constexpr TwoCfg kTwoKV{DC_TWO_NT_KV, DC_TWO_IT_KV};
constexpr TwoCfg kTwoF32{DC_TWO_NT, DC_TWO_IT};   // f32 keys: stable merges
constexpr int kTwoMinT = cmin(cmin(kTwoKeys.T(), kTwoKV.T()), kTwoF32.T());
template <class K, bool V>
constexpr TwoCfg two_cfg() { return V ? kTwoKV : (K::kNeedStable ? kTwoF32 : kTwoKeys); }

size_t two_level_tab_entries(int64_t) { return 0; }
size_t two_level_bnd_entries(int64_t n) {
    // groups at the smallest width (w = tile, any configuration) have the most tiles
    const int64_t w = kMinTile;
    const int64_t groups = (n + 4 * w - 1) / (4 * w);
    return 4 * ((size_t)(groups * num_tiles(4 * w, kTwoMinT)) + 2);
}

size_t scratch_needed(int64_t n, bool vals) {
    size_t kb = align_up((size_t)n * 4, 256);
    return kb + (vals ? kb : 0) + align_up(split_entries(n) * 4, 256) +
           align_up(two_level_tab_entries(n) * 4, 256) + align_up(two_level_bnd_entries(n) * 4, 256);
}

dc_status check_plan(dc_plan_t p) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (p->bad) return fail(DC_ERR_BAD_STATE, "plan poisoned by an earlier CUDA error");
    return DC_OK;
}

dc_status cuda_fail(dc_plan_t p, cudaError_t e, const char* what) {
    if (p) p->bad = true;
    return fail(DC_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

#define DC_CUDA(p, call)                                          \
    do {                                                          \
        cudaError_t e_ = (call);                                  \
        if (e_ != cudaSuccess) return cuda_fail((p), e_, #call);  \
    } while (0)

#define DC_LAUNCHED(p)                                                     \
    do {                                                                   \
        cudaError_t e_ = cudaGetLastError();                               \
        if (e_ != cudaSuccess) return cuda_fail((p), e_, "kernel launch"); \
        (p)->launches++;                                                   \
    } while (0)

cudaEvent_t take_event(dc_plan_t p) {
    if (!p->event_pool.empty()) {
        cudaEvent_t e = p->event_pool.back();
        p->event_pool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
}

// Brackets one kernel launch with events on the plan stream when timing is on.
struct TimedScope {
    dc_plan_t p;
    int kind;
    cudaStream_t s;
    cudaEvent_t e0 = nullptr;
    TimedScope(dc_plan_t p_, int kind_) : TimedScope(p_, kind_, p_->stream) {}
    TimedScope(dc_plan_t p_, int kind_, cudaStream_t s_) : p(p_), kind(kind_), s(s_) {
        if (p->timing) {
            e0 = take_event(p);
            cudaEventRecord(e0, s);
        }
    }
    ~TimedScope() {
        if (e0) {
            cudaEvent_t e1 = take_event(p);
            cudaEventRecord(e1, s);
            p->pending.push_back({kind, e0, e1});
        }
    }
};

bool aligned16(const void* ptr) { return ((uintptr_t)ptr & 15u) == 0; }

// Captured sort graphs embed the plan's scratch / staging / slot pointers, so
// every reallocation of one of them drops the cache (a graph
// replayed after a larger run reallocated scratch read freed memory).
void drop_graphs(dc_plan_t p) {
    for (auto& gc : p->graphs) {
        if (gc.exec) cudaGraphExecDestroy(gc.exec);
        if (gc.graph) cudaGraphDestroy(gc.graph);
    }
    p->graphs.clear();
}

// Per-device, thread-safe one-time setup (kernel attributes, occupancy
// grids): the dynamic shared-memory attribute and the occupancy are
// properties of (function, device), so a cache keyed only by the
// instantiation would skip the attribute on a second GPU of the process.
constexpr int kMaxDevices = 64;
int current_device() {
    int d = 0;
    cudaGetDevice(&d);
    return d < 0 ? 0 : (d >= kMaxDevices ? kMaxDevices - 1 : d);
}
struct PerDevice {
    std::atomic<int> v[kMaxDevices];
    int get() const { return v[current_device()].load(std::memory_order_acquire); }
    void set(int x) { v[current_device()].store(x, std::memory_order_release); }
};

// Orders a run on the plan stream after every host-buffer sort submitted
// before it (those run on p->comp and share the plan scratch).
dc_status join_host_sorts(dc_plan_t p) {
    if (p->comp && p->comp_done && p->stream != p->comp) {
        cudaError_t e = cudaStreamWaitEvent(p->stream, p->comp_done, 0);
        if (e != cudaSuccess) return cuda_fail(p, e, "cudaStreamWaitEvent(host sorts)");
    }
    return DC_OK;
}

dc_status ensure_scratch(dc_plan_t p, bool vals) {
    size_t need = scratch_needed(p->n, vals);
    if (p->scratch && p->scratch_bytes >= need) return DC_OK;
    if (p->scratch && !p->own_scratch)
        return fail(DC_ERR_INVALID_ARG, "caller scratch too small for this run");
    drop_graphs(p);
    if (p->scratch) {
        cudaFree(p->scratch);
        p->scratch = nullptr;
    }
    void* ptr = nullptr;
    cudaError_t e = cudaMalloc(&ptr, need);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(DC_ERR_OUT_OF_MEMORY, "scratch cudaMalloc failed");
    }
    p->scratch = ptr;
    p->scratch_bytes = need;
    p->own_scratch = true;
    return DC_OK;
}

dc_status ensure_pipeline(dc_plan_t p, int chunks) {
    while ((int)p->pipe_streams.size() < chunks) {
        cudaStream_t st = nullptr;
        DC_CUDA(p, cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
        p->pipe_streams.push_back(st);
    }
    while ((int)p->pipe_events.size() < chunks + 1) {
        cudaEvent_t ev = nullptr;
        DC_CUDA(p, cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        p->pipe_events.push_back(ev);
    }
    return DC_OK;
}

// One two-level pass (f1) over the runs P describes: the exact 4-run cuts of
// every output tile (nk2_select4), then the persistent 4-way tile merge
// (nk3_merge4) into dst.  Used by the breadth-first sort (uniform groups of
// four runs) and by the multi-GPU G-way merge (one custom group per launch).
template <class K, bool V>
dc_status pass4(dc_plan_t p, const dc::Pass4& P, int tiles, dc::Cut4* cuts, uint32_t* dst_k,
                uint32_t* dst_v, cudaStream_t st) {
    constexpr TwoCfg TC = two_cfg<K, V>();
    auto* k32 = dc::nk3_merge4<TC.nt, TC.it, K, V>;
    constexpr int thr2 = TC.threads();
    constexpr int smem2 = dc::m4_smem_bytes(TC.T(), TC.it, V);
    static PerDevice grid2_dev;                  // per instantiation and device
    int grid2 = grid2_dev.get();
    if (!grid2) {
        DC_CUDA(p, cudaFuncSetAttribute(k32, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2));
        int dev = 0, sms = 148, occ = 1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k32, thr2, smem2);
        grid2 = sms * (occ > 0 ? occ : 1);
        grid2_dev.set(grid2);
    }
    if (tiles <= 0) return DC_OK;
    {
        TimedScope ts(p, DC_KERNEL_NK2_PARTITION, st);
#ifndef DC_SEL4_PV_KV
#define DC_SEL4_PV_KV 2   // r02b: 0.689 -> 0.652 ms per 2^28 key-value sort (PV 4 before the branch-free rounds)
#endif
#ifndef DC_SEL4_PV_KEYS
#define DC_SEL4_PV_KEYS 2
#endif
        constexpr int PV = V ? DC_SEL4_PV_KV : DC_SEL4_PV_KEYS;   // pivots per run (sort4_kernels.cuh)
        constexpr int bpw = dc::sel4_bpw<PV>();
        const int sel_warps = (tiles + bpw - 1) / bpw;
        dc::nk2_select4<K, PV><<<(sel_warps + 3) / 4, 128, 0, st>>>(P, tiles, cuts);
        DC_LAUNCHED(p);
    }
    {
        TimedScope ts(p, DC_KERNEL_NK3_MERGE, st);
        k32<<<std::min(tiles, grid2), thr2, smem2, st>>>(P, dst_k, dst_v, cuts, tiles);
        DC_LAUNCHED(p);
    }
    return DC_OK;
}

// Sorts keys[0..n) (+ vals) into out_k (+ out_v); out may equal the input
// (in place).  NK1 reads the input; the passes ping-pong between scratch and
// the output buffer.
template <class K, bool V, bool SMALL>
dc_status sort_typed(dc_plan_t p, uint32_t* keys, uint32_t* vals, uint32_t* out_k,
                     uint32_t* out_v, bool two_level, int cs) {
    const int64_t n = p->n;
    const bool hv = V;
    dc_status st = ensure_scratch(p, hv);
    if (st != DC_OK) return st;
    size_t kb = align_up((size_t)n * 4, 256);
    uint32_t* sk = (uint32_t*)p->scratch;
    uint32_t* sv = hv ? (uint32_t*)((char*)p->scratch + kb) : nullptr;
    int* split = (int*)((char*)p->scratch + kb + (hv ? kb : 0));

    constexpr SortCfg C = cfg_for<K, V, SMALL>();
    auto* k1 = dc::nk1_blocksort<C.nt1, C.it1, K, V>;
    auto* k3 = dc::nk3_merge<C.nt3, C.it, K, V>;
    auto* k3sp = dc::nk3_merge_sp<C.nt3, C.it, K, V>;   // partition fused (SMALL)
    static PerDevice attr_done;   // per instantiation and device
    if (!attr_done.get()) {
        DC_CUDA(p, cudaFuncSetAttribute(k1, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        nk1_smem_bytes(C, hv)));
        DC_CUDA(p, cudaFuncSetAttribute(k3, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        nk3_smem_bytes(C, hv)));
        if (SMALL)
            DC_CUDA(p, cudaFuncSetAttribute(k3sp, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                            nk3_smem_bytes(C, hv)));
        attr_done.set(1);
    }

    // Levels over HBM: P = ceil(log2(ceil(n/tile))).  Keys-only sorts fold
    // two levels into one pass (4-way groups, sort4_kernels.cuh); with P odd
    // one single-level pass goes first.
    // f2: NK1 cluster levels (keys-only u32/i32): the fused runs are cs tiles wide.
    constexpr bool kClCapable = !V && !K::kNeedStable;
    if (!kClCapable) cs = 1;
    const bool kCl = cs > 1;
    const int64_t ftile = (int64_t)C.tile() * cs;
    const int P = global_passes(n, ftile);
    constexpr bool kTwoCapable = true;
    const bool two = two_level && P >= 2;
    const int single = two ? (P % 2) : P;
    const int passes = two ? single + (P - single) / 2 : P;
    // Ping-pong parity: the last pass must write the output buffer, so NK1
    // writes the output buffer iff the number of passes is even.
    uint32_t* cur_k = (passes % 2 == 0) ? out_k : sk;
    uint32_t* cur_v = (passes % 2 == 0) ? out_v : sv;
    uint32_t* oth_k = (passes % 2 == 0) ? sk : out_k;
    uint32_t* oth_v = (passes % 2 == 0) ? sv : out_v;

    // One merge level over [org, end) on stream `st` (split region `sp`).
    auto level = [&](int64_t org, int64_t end, int64_t w, int* sp, cudaStream_t st) -> dc_status {
        const int tpg = (int)num_tiles(std::min<int64_t>(2 * w, end - org), C.tout());
        const int tiles = (int)(num_tiles(end - org, 2 * w) * tpg);
        const dc::PairGeom g{org, w, w, end, tpg};
        if (SMALL && p->fuse_partition) {
            // L2-resident: every merge CTA finds its own co-ranks (one launch per level)
            TimedScope ts(p, DC_KERNEL_NK3_MERGE, st);
            k3sp<<<tiles, C.nt3, nk3_smem_bytes(C, hv), st>>>(cur_k, cur_v, oth_k, oth_v, g);
            DC_LAUNCHED(p);
            return DC_OK;
        }
        {
            TimedScope ts(p, DC_KERNEL_NK2_PARTITION, st);
#ifndef DC_NK2_WARP_ALL
#define DC_NK2_WARP_ALL 0
#endif
            if (SMALL || DC_NK2_WARP_ALL)   // L2-resident: 33-ary warp searches, few dependent rounds
                dc::nk2_partition_warp<K><<<(tiles + 3) / 4, 128, 0, st>>>(cur_k, g, C.tout(),
                                                                         tiles, sp);
            else
                dc::nk2_partition<K><<<(tiles + 255) / 256, 256, 0, st>>>(cur_k, g, C.tout(),
                                                                         tiles, sp);
            DC_LAUNCHED(p);
        }
        {
            TimedScope ts(p, DC_KERNEL_NK3_MERGE, st);
            k3<<<tiles, C.nt3, nk3_smem_bytes(C, hv), st>>>(cur_k, cur_v, oth_k, oth_v, sp, g);
            DC_LAUNCHED(p);
        }
        return DC_OK;
    };

    int64_t w = ftile;
    int lv = 0;
    // Chunked pipeline (one-level schedule, not while timing kernels): the
    // bottom `lc` levels of every chunk of tile*2^lc keys run on the chunk's
    // own stream right after its NK1; chunks overlap each other.
    int lc = 0, chunks = 1;
    if (!SMALL && !kCl && !two && !p->timing && p->pipe_chunks > 1) {
        int lt = 0;
        while ((1 << lt) < p->pipe_chunks) ++lt;
        if (single > lt) {
            lc = single - lt;
            chunks = (int)num_tiles(n, (int64_t)C.tile() << lc);
        }
    }
    if (chunks > 1) {
        st = ensure_pipeline(p, chunks);
        if (st != DC_OK) return st;
        const int64_t clen = (int64_t)C.tile() << lc;
        const size_t split_per = (size_t)num_tiles(clen, C.tout()) + (size_t)num_tiles(clen, 2 * (int64_t)C.tile()) + 2;
        DC_CUDA(p, cudaEventRecord(p->pipe_events[0], p->stream));
        for (int c = 0; c < chunks; ++c) {
            cudaStream_t cs = p->pipe_streams[c];
            const int64_t org = c * clen, end = std::min(n, org + clen);
            DC_CUDA(p, cudaStreamWaitEvent(cs, p->pipe_events[0], 0));
            {
                TimedScope ts(p, DC_KERNEL_NK1_BLOCKSORT, cs);
                k1<<<(unsigned)num_tiles(end - org, C.tile()), C.nt1, nk1_smem_bytes(C, hv), cs>>>(
                    keys + org, vals ? vals + org : nullptr, cur_k + org,
                    cur_v ? cur_v + org : nullptr, end - org);
                DC_LAUNCHED(p);
            }
            uint32_t *ck = cur_k, *cv = cur_v, *ok = oth_k, *ov = oth_v;
            for (int l = 0; l < lc; ++l) {
                st = level(org, end, (int64_t)C.tile() << l, split + c * split_per, cs);
                if (st != DC_OK) return st;
                std::swap(cur_k, oth_k);
                std::swap(cur_v, oth_v);
            }
            cur_k = ck; cur_v = cv; oth_k = ok; oth_v = ov;   // same parity for every chunk
            DC_CUDA(p, cudaEventRecord(p->pipe_events[1 + c], cs));
        }
        for (int c = 0; c < chunks; ++c)
            DC_CUDA(p, cudaStreamWaitEvent(p->stream, p->pipe_events[1 + c], 0));
        for (int l = 0; l < lc; ++l) {
            std::swap(cur_k, oth_k);
            std::swap(cur_v, oth_v);
        }
        w = (int64_t)C.tile() << lc;
        lv = lc;
    } else {
        // NK1: base cases + fused bottom levels (reads the caller's buffer).
        TimedScope ts(p, DC_KERNEL_NK1_BLOCKSORT);
        if (kCl) {
            if constexpr (kClCapable) {
                auto* kc = dc::nk1_blocksort_cl<C.nt1, C.it1, K>;
                const int smem = dc::tile_words(C.tile(), C.it1 + 4) * 4;
                static PerDevice cl_attr;
                if (!cl_attr.get()) {
                    DC_CUDA(p, cudaFuncSetAttribute(kc, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
                    DC_CUDA(p, cudaFuncSetAttribute(kc, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
                    cl_attr.set(1);
                }
                cudaLaunchConfig_t cfg = {};
                cfg.gridDim = dim3((unsigned)(num_tiles(n, ftile) * cs));
                cfg.blockDim = dim3(C.nt1);
                cfg.dynamicSmemBytes = (size_t)smem;
                cfg.stream = p->stream;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeClusterDimension;
                at[0].val.clusterDim.x = (unsigned)cs;
                at[0].val.clusterDim.y = 1;
                at[0].val.clusterDim.z = 1;
                cfg.attrs = at;
                cfg.numAttrs = 1;
                DC_CUDA(p, cudaLaunchKernelEx(&cfg, kc, (const uint32_t*)keys, cur_k, (long long)n));
            }
        } else {
            k1<<<(unsigned)num_tiles(n, C.tile()), C.nt1, nk1_smem_bytes(C, hv), p->stream>>>(
                keys, vals, cur_k, cur_v, n);
        }
        DC_LAUNCHED(p);
    }
#ifdef DC_ONLY_NK1   // measurement builds only: time the fused kernel alone
    return DC_OK;
#endif
    for (; lv < single; ++lv, w *= 2) {
        st = level(0, n, w, split, p->stream);
        if (st != DC_OK) return st;
        std::swap(cur_k, oth_k);
        std::swap(cur_v, oth_v);
    }
    if constexpr (kTwoCapable) {
        if (two) {
            int* tab = split + align_up(split_entries(n) * 4, 256) / 4;
            dc::Cut4* cuts = (dc::Cut4*)(tab + align_up(two_level_tab_entries(n) * 4, 256) / 4);
            for (; w < n; w *= 4) {
                const int tpg = (int)num_tiles(std::min<int64_t>(4 * w, n), two_cfg<K, V>().T());
                dc::Pass4 P{};
                for (int q = 0; q < 4; ++q) {
                    P.k[q] = cur_k;
                    P.v[q] = cur_v;
                    P.bound[q] = n;
                }
                P.n = n;
                P.w = w;
                P.T = two_cfg<K, V>().T();
                P.tpg = tpg;
                P.custom = 0;
                const int tiles2 = (int)(((n + 4 * w - 1) / (4 * w)) * tpg);
                st = pass4<K, V>(p, P, tiles2, cuts, oth_k, oth_v, p->stream);
                if (st != DC_OK) return st;
                std::swap(cur_k, oth_k);
                std::swap(cur_v, oth_v);
            }
        }
    }
    return DC_OK;
}

// The schedule of one sort: the planner's choice (model.cu, dc_model_sort_
// schedule) among the compiled tile classes and pass kinds, unless the plan
// forces one of them.
struct Decision {
    bool small, two;
    int cs;   // NK1 cluster size (1: plain NK1)
};
// NK1 cluster rule (keys-only u32/i32).  Measured r02b (tools/cluster_sweep.py,
// profiles/r02b/cluster_sweep.txt: u32, n = 2^16..2^26, cs = 1..16, both tile
// classes and pass kinds): a cluster level costs about what the global level it
// removes costs at small n (both latency-bound, ~5-8 us) and more at large n
// (0.40 vs 0.26 ms per level at 2^28): no size gains more than one ~2 us
// timer quantum (2^18: cs = 8 57.3 vs 59.4 us), most lose.  The rule keeps
// them off; dc_plan_set_nk1_cluster forces them.
int cluster_rule(int64_t, bool) { return 1; }
Decision decide(dc_plan_t p, dc_key_type kt, bool vals) {
    dc_sort_schedule s{};
    dc_model_sort_schedule(p->n, kt, vals ? 1 : 0, p->tile_class, p->two_force, &s);
    const bool small = s.tile_class == 1;
    int cs = 1;
    if (!vals && kt != DC_KEY_F32) cs = p->nk1_cluster ? p->nk1_cluster : cluster_rule(p->n, small);
    return {small, s.two_level != 0, cs};
}

template <class K>
dc_status sort_kv_dispatch(dc_plan_t p, dc_key_type kt, uint32_t* keys, uint32_t* vals,
                           uint32_t* ok, uint32_t* ov) {
    const Decision d = decide(p, kt, vals != nullptr);
    if (vals) return d.small ? sort_typed<K, true, true>(p, keys, vals, ok, ov, d.two, 1)
                             : sort_typed<K, true, false>(p, keys, vals, ok, ov, d.two, 1);
    return d.small ? sort_typed<K, false, true>(p, keys, nullptr, ok, nullptr, d.two, d.cs)
                   : sort_typed<K, false, false>(p, keys, nullptr, ok, nullptr, d.two, d.cs);
}

dc_status sort_direct(dc_plan_t p, dc_key_type kt, uint32_t* keys, uint32_t* vals, uint32_t* ok,
                      uint32_t* ov) {
    switch (kt) {
        case DC_KEY_U32: return sort_kv_dispatch<dc::KeyU32>(p, kt, keys, vals, ok, ov);
        case DC_KEY_I32: return sort_kv_dispatch<dc::KeyI32>(p, kt, keys, vals, ok, ov);
        case DC_KEY_F32: return sort_kv_dispatch<dc::KeyF32>(p, kt, keys, vals, ok, ov);
    }
    return fail(DC_ERR_INVALID_ARG, "unknown key type");
}

// CUDA-graph replay of the whole level sequence (launch-bound small sorts).
// The first run for a given (keys, vals, key type) executes eagerly (it
// allocates scratch and sets kernel attributes); the second captures the
// launches on a plan-owned stream and instantiates a graph; later runs
// replay it on the plan stream.  Off while per-kernel timing is enabled.
dc_status sort_dispatch(dc_plan_t p, dc_key_type kt, uint32_t* keys, uint32_t* vals,
                        uint32_t* ok = nullptr, uint32_t* ov = nullptr) {
    if (!ok) {                                   // in place
        ok = keys;
        ov = vals;
    }
    dc_status js = join_host_sorts(p);
    if (js != DC_OK) return js;
    if (!p->use_graphs || p->timing) return sort_direct(p, kt, keys, vals, ok, ov);
    for (auto& gc : p->graphs) {
        if (gc.keys == keys && gc.vals == vals && gc.out == ok && gc.kt == kt) {
            if (!gc.exec) {                                   // second sighting: capture
                if (!p->cap_stream)
                    DC_CUDA(p, cudaStreamCreateWithFlags(&p->cap_stream, cudaStreamNonBlocking));
                cudaStream_t user = p->stream;
                p->stream = p->cap_stream;
                DC_CUDA(p, cudaStreamBeginCapture(p->cap_stream, cudaStreamCaptureModeThreadLocal));
                const int64_t l0 = p->launches;
                dc_status st = sort_direct(p, kt, keys, vals, ok, ov);
                cudaGraph_t graph = nullptr;
                cudaError_t e = cudaStreamEndCapture(p->cap_stream, &graph);
                p->stream = user;
                if (st != DC_OK) return st;
                if (e != cudaSuccess) return cuda_fail(p, e, "cudaStreamEndCapture");
                gc.graph = graph;
                gc.launches = p->launches - l0;
                p->launches = l0;
                DC_CUDA(p, cudaGraphInstantiate(&gc.exec, graph, 0));
            }
            DC_CUDA(p, cudaGraphLaunch(gc.exec, p->stream));
            p->launches += gc.launches;
            return DC_OK;
        }
    }
    if (p->graphs.size() >= 8) return sort_direct(p, kt, keys, vals, ok, ov);
    p->graphs.push_back({keys, vals, ok, kt, nullptr, nullptr, 0});   // first sighting: eager
    return sort_direct(p, kt, keys, vals, ok, ov);
}

// Max-subarray kernel: DC_MS_TMA = 1 (default) streams every lane's range by
// TMA (maxsub_tma.cuh, one CTA per SM); 0 is the register-load version.
#ifndef DC_MS_TMA
#define DC_MS_TMA 1
#endif
#ifndef DC_MS_P            // L: elements per lane per warp segment (L/4 odd); r02b: 68 -> 76
#define DC_MS_P 76
#endif
#ifndef DC_MS_S
#define DC_MS_S 2
#endif
#ifndef DC_MS_TNT
#define DC_MS_TNT 256
#endif
#ifndef DC_MS_J
#define DC_MS_J 2
#endif
// Values-only element fold + chunk-label index recovery (DESIGN R21).  r02b:
// default once the recovery became warp-parallel and the trees branch-free
// (2^24: 26.86 us indexed fold, L = 68 -> 24.93 us values-only, L = 76; 50
// steps each, profiles/r02b/nk4_sweep.txt); 0 keeps the indexed fold.
#ifndef DC_MS_VONLY
#define DC_MS_VONLY 1
#endif
// DC_MS_ROWS = 1: every lane folds one contiguous row, rows fed by 2-D TMA
// tensor copies, 3 CTAs per SM (maxsub_rows.cuh).  Measured at 2^24 (r02,
// profiles/r02/nk4_variants.txt): 28.9-33.3 us per launch over five ring
// shapes against 28.8 us for the warp-segment kernel (0, default): tripling
// the resident warps did not raise the issue rate (52 %), the per-element fold
// (~17 instructions, selects on the half-rate ALU pipe) bounds both.
#ifndef DC_MS_ROWS
#define DC_MS_ROWS 0
#endif
#ifndef DC_MS_RNT          // rows kernel: threads per CTA
#define DC_MS_RNT 256
#endif
#ifndef DC_MS_RL           // columns per TMA box (L/4 odd)
#define DC_MS_RL 28
#endif
#ifndef DC_MS_RS           // ring stages
#define DC_MS_RS 2
#endif
#ifndef DC_MS_RMINB        // CTAs per SM the register budget is sized for
#define DC_MS_RMINB 3
#endif
constexpr int kMsRNT = DC_MS_RNT, kMsRL = DC_MS_RL, kMsRS = DC_MS_RS, kMsRMinB = DC_MS_RMINB;
constexpr int ms_rows_smem() { return kMsRS * kMsRNT * kMsRL * 4; }   // S x NW x 32 x L words
constexpr int kMsP = DC_MS_P, kMsS = DC_MS_S, kMsTNT = DC_MS_TNT, kMsJ = DC_MS_J;
constexpr bool kMsVO = DC_MS_VONLY != 0;
constexpr int ms_tma_smem() { return kMsS * kMsTNT * kMsP * 4; }   // S x NW x 32*L words

// Max-subarray grid: about one wave of resident CTAs (occupancy x SMs),
// never more CTAs than there is work for.
int ms_grid(dc_plan_t p) {
    static PerDevice grid_dev;
    int grid = grid_dev.get();
    if (!grid) {
        int dev = 0, sms = 148, occ = 1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (DC_MS_ROWS) {
            auto* k = dc::nk4_maxsub_rows<kMsRNT, kMsRL, kMsRS, kMsRMinB>;
            cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, ms_rows_smem());
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, kMsRNT, ms_rows_smem());
        } else if (DC_MS_TMA) {
            auto* k = dc::nk4_maxsub_tma<kMsTNT, kMsP, kMsS, kMsJ, kMsVO>;
            cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, ms_tma_smem());
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, kMsTNT, ms_tma_smem());
        } else {
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(
                &occ, dc::nk4_maxsub<kNK4Threads, kNK4Chunk>, kNK4Threads, 0);
        }
        grid = sms * (occ > 0 ? occ : 1);
        grid_dev.set(grid);
    }
    const int64_t units = DC_MS_ROWS ? num_tiles(p->n, (int64_t)kMsRNT * kMsRL)   // rows >= L
                          : DC_MS_TMA ? num_tiles(p->n, (int64_t)kMsTNT * kMsP)   // >= 1 segment/warp
                                      : num_tiles(p->n, kMsTile);
    return (int)(units < grid ? units : grid);
}

dc_status ensure_ms_state(dc_plan_t p) {
    if (p->ms_tiles) return DC_OK;
    const size_t parts = (size_t)ms_grid(p);
    void* ptr = nullptr;
    const size_t bytes = align_up(parts * sizeof(dc_maxsub_tuple), 256) + 256 + 256;
    if (cudaMalloc(&ptr, bytes) != cudaSuccess) {
        cudaGetLastError();
        return fail(DC_ERR_OUT_OF_MEMORY, "max-subarray state cudaMalloc failed");
    }
    DC_CUDA(p, cudaMemsetAsync(ptr, 0, bytes, p->stream));
    p->ms_tiles = (dc_maxsub_tuple*)ptr;
    p->ms_ticket = (unsigned int*)((char*)ptr + align_up(parts * sizeof(dc_maxsub_tuple), 256));
    p->ms_res = (dc_maxsub_result*)((char*)p->ms_ticket + 256);
    return DC_OK;
}

dc_status maxsub_launch(dc_plan_t p, const int32_t* d_x, int64_t off, int mode,
                        dc_maxsub_result* out_res, dc_maxsub_tuple* out_tup) {
    dc_status st = ensure_ms_state(p);
    if (st != DC_OK) return st;
    const int grid = ms_grid(p);
    if (DC_MS_ROWS) {
        // rows of W elements (16-byte multiple), one per lane of the grid
        const int64_t lanes = (int64_t)grid * kMsRNT;
        int64_t W = (p->n + lanes - 1) / lanes;
        W = std::max<int64_t>(4, (W + 3) / 4 * 4);
        if (W > 65536) return fail(DC_ERR_UNSUPPORTED, "max-subarray rows longer than 2^16");
        const dc::MsRows g{p->n, W, p->n / W};
        if (p->ms_map_x != (const void*)d_x || p->ms_map_n != p->n || p->ms_map_w != W) {
            std::memset(&p->ms_map, 0, sizeof(p->ms_map));
            if (g.nrows > 0) {
                static PFN_cuTensorMapEncodeTiled_v12000 encode = [] {
                    void* fn = nullptr;
                    cudaDriverEntryPointQueryResult q;
                    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault,
                                                &q) != cudaSuccess ||
                        q != cudaDriverEntryPointSuccess) {
                        cudaGetLastError();
                        fn = nullptr;
                    }
                    return (PFN_cuTensorMapEncodeTiled_v12000)fn;
                }();
                if (!encode) return fail(DC_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
                const cuuint64_t dims[2] = {(cuuint64_t)W, (cuuint64_t)g.nrows};
                const cuuint64_t strides[1] = {(cuuint64_t)W * 4};
                const cuuint32_t box[2] = {(cuuint32_t)kMsRL, 32};
                const cuuint32_t estr[2] = {1, 1};
                const CUresult r = encode(&p->ms_map, CU_TENSOR_MAP_DATA_TYPE_INT32, 2,
                                          const_cast<int32_t*>(d_x), dims, strides, box, estr,
                                          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                          CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
                if (r != CUDA_SUCCESS) return fail(DC_ERR_CUDA, "cuTensorMapEncodeTiled failed");
            }
            p->ms_map_x = d_x;
            p->ms_map_n = p->n;
            p->ms_map_w = W;
        }
        TimedScope ts(p, DC_KERNEL_NK4_MAXSUB);
        dc::nk4_maxsub_rows<kMsRNT, kMsRL, kMsRS, kMsRMinB>
            <<<grid, kMsRNT, ms_rows_smem(), p->stream>>>(p->ms_map, d_x, g, p->ms_tiles,
                                                          p->ms_ticket, off, mode, out_res, out_tup);
        DC_LAUNCHED(p);
        return DC_OK;
    }
    TimedScope ts(p, DC_KERNEL_NK4_MAXSUB);
    if (DC_MS_TMA) {
        // warp ranges of RW elements, a multiple of the 32*L-element segment
        const int64_t warps = (int64_t)grid * (kMsTNT / 32), seg = 32LL * kMsP;
        const int64_t R = ((p->n + warps - 1) / warps + seg - 1) / seg * seg;
        dc::nk4_maxsub_tma<kMsTNT, kMsP, kMsS, kMsJ, kMsVO><<<grid, kMsTNT, ms_tma_smem(), p->stream>>>(
            d_x, p->n, R, p->ms_tiles, p->ms_ticket, off, mode, out_res, out_tup);
    } else {
        dc::nk4_maxsub<kNK4Threads, kNK4Chunk><<<grid, kNK4Threads, 0, p->stream>>>(
            d_x, p->n, p->ms_tiles, p->ms_ticket, off, mode, out_res, out_tup);
    }
    DC_LAUNCHED(p);
    return DC_OK;
}

dc_status ensure_stage(dc_plan_t p, size_t bytes) {
    if (p->d_stage && p->d_stage_bytes >= bytes) return DC_OK;
    drop_graphs(p);
    if (p->d_stage) cudaFree(p->d_stage);
    p->d_stage = nullptr;
    if (cudaMalloc(&p->d_stage, bytes) != cudaSuccess) {
        cudaGetLastError();
        p->d_stage = nullptr;
        return fail(DC_ERR_OUT_OF_MEMORY, "staging cudaMalloc failed");
    }
    p->d_stage_bytes = bytes;
    return DC_OK;
}


// a9: local stable G-way merge (Alg 7's top log2 G levels, earlier runs win
// ties).  A run is (key buffer, value buffer, readable length, offset,
// length); in the first round the buffers may be peer GPUs' sorted shards
// (the fused exchange) or the all-to-all receive buffer.  Every round merges
// consecutive groups of FOUR runs with one two-level pass each (f1's exact
// 4-run selection + 4-way tile merge, Pass4 custom mode), a trailing group of
// two with one pair-mode merge pass (NK2 co-ranks + NK3 tiles over separately
// addressed runs), a lone run by a copy; the merged groups are the next
// round's runs.  HBM passes: ceil(log4 G) -- G = 2..4: one, G = 5..16: two --
// against ceil(log2 G) for pairwise rounds.  Rounds write d0, d1, d0, ... and
// the last one the output buffers.
struct RunRef {
    const uint32_t* k;
    const uint32_t* v;
    int64_t bound, off, len;
};

template <class K, bool V>
dc_status merge_g(dc_plan_t p, std::vector<RunRef> runs, uint32_t* d0_k, uint32_t* d0_v,
                  uint32_t* d1_k, uint32_t* d1_v, uint32_t* out_k, uint32_t* out_v) {
    int64_t total = 0;
    for (const RunRef& r : runs) total += r.len;
    if (total > p->n) return fail(DC_ERR_INVALID_ARG, "runs exceed the plan size");
    dc_status st = join_host_sorts(p);
    if (st != DC_OK) return st;
    st = ensure_scratch(p, V);
    if (st != DC_OK) return st;
    const size_t kb = align_up((size_t)p->n * 4, 256);
    int* split = (int*)((char*)p->scratch + kb + (V ? kb : 0));
    dc::Cut4* cuts = (dc::Cut4*)(split + align_up(split_entries(p->n) * 4, 256) / 4 +
                                 align_up(two_level_tab_entries(p->n) * 4, 256) / 4);
    constexpr SortCfg C = cfg_for<K, V, false>();
    constexpr int T4 = two_cfg<K, V>().T();
    auto* k3 = dc::nk3_merge_ab<C.nt3, C.it, K, V>;
    static PerDevice attr_done;
    if (!attr_done.get()) {
        DC_CUDA(p, cudaFuncSetAttribute(k3, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        nk3_smem_bytes(C, V)));
        attr_done.set(1);
    }
    if (runs.empty()) return DC_OK;
    int rounds = 0;
    for (size_t c = runs.size(); c > 1; c = (c + 3) / 4) ++rounds;
    if (rounds == 0) rounds = 1;                       // a single run: one copy round
    for (int rd = 0; rd < rounds; ++rd) {
        const bool last = rd == rounds - 1;
        uint32_t* dk = last ? out_k : (rd % 2 == 0 ? d0_k : d1_k);
        uint32_t* dv = last ? out_v : (rd % 2 == 0 ? d0_v : d1_v);
        std::vector<RunRef> next;
        int64_t org = 0;
        for (size_t g = 0; g < runs.size(); g += 4) {
            const size_t cnt = std::min<size_t>(4, runs.size() - g);
            int64_t glen = 0;
            for (size_t q = 0; q < cnt; ++q) glen += runs[g + q].len;
            if (glen > 0 && cnt >= 3) {                 // two levels in one pass
                dc::Pass4 P{};
                for (int q = 0; q < 4; ++q) {
                    const RunRef& r = runs[g + std::min<size_t>(q, cnt - 1)];
                    P.k[q] = r.k;
                    P.v[q] = r.v;
                    P.bound[q] = r.bound;
                    P.off[q] = r.off;
                    P.len[q] = (size_t)q < cnt ? r.len : 0;
                }
                P.out0 = org;
                P.T = T4;
                P.tpg = (int)num_tiles(glen, T4);
                P.custom = 1;
                st = pass4<K, V>(p, P, P.tpg, cuts, dk, dv, p->stream);
                if (st != DC_OK) return st;
            } else if (glen > 0 && cnt == 2) {          // one level
                const RunRef& A = runs[g];
                const RunRef& B = runs[g + 1];
                const int tiles = (int)num_tiles(glen, C.tout());
                {
                    TimedScope ts(p, DC_KERNEL_NK2_PARTITION);
                    dc::nk2_partition_ab<K><<<(tiles + 3) / 4, 128, 0, p->stream>>>(
                        A.k + A.off, A.len, B.k + B.off, B.len, C.tout(), tiles, split);
                    DC_LAUNCHED(p);
                }
                {
                    TimedScope ts(p, DC_KERNEL_NK3_MERGE);
                    k3<<<tiles, C.nt3, nk3_smem_bytes(C, V), p->stream>>>(
                        A.k, A.v, A.bound, A.off, A.len, B.k, B.v, B.bound, B.off, B.len, dk, dv,
                        org, split);
                    DC_LAUNCHED(p);
                }
            } else if (glen > 0) {                      // a lone run moves as it is
                const RunRef& A = runs[g];
                DC_CUDA(p, cudaMemcpyAsync(dk + org, A.k + A.off, (size_t)A.len * 4,
                                           cudaMemcpyDeviceToDevice, p->stream));
                if (V)
                    DC_CUDA(p, cudaMemcpyAsync(dv + org, A.v + A.off, (size_t)A.len * 4,
                                               cudaMemcpyDeviceToDevice, p->stream));
            }
            next.push_back({dk, dv, total, org, glen});
            org += glen;
        }
        runs.swap(next);
    }
    return DC_OK;
}

// dc_mg_merge_runs: back-to-back runs of one buffer; intermediate rounds
// ping-pong between the plan scratch and the (clobbered) input.
template <class K, bool V>
dc_status mg_merge_typed(dc_plan_t p, uint32_t* in_k, uint32_t* in_v, uint32_t* out_k,
                         uint32_t* out_v, const std::vector<int64_t>& lens) {
    int64_t total = 0;
    for (int64_t l : lens) total += l;
    std::vector<RunRef> runs;
    int64_t org = 0;
    for (int64_t l : lens) {
        runs.push_back({in_k, in_v, total, org, l});
        org += l;
    }
    dc_status st = ensure_scratch(p, V);
    if (st != DC_OK) return st;
    const size_t kb = align_up((size_t)p->n * 4, 256);
    uint32_t* sk = (uint32_t*)p->scratch;
    uint32_t* sv = V ? (uint32_t*)((char*)p->scratch + kb) : nullptr;
    return merge_g<K, V>(p, runs, sk, sv, in_k, in_v, out_k, out_v);
}

// a8+a9 fused (dc_mg_merge_peers): the first round reads the runs where they
// lie (peer shards over NVLink); later rounds are local (tmp, then scratch).
template <class K, bool V>
dc_status mg_merge_peers_typed(dc_plan_t p, const uint32_t* const* rk, const uint32_t* const* rv,
                               const int64_t* bound, const int64_t* off, const int64_t* len,
                               int runs, uint32_t* tmp_k, uint32_t* tmp_v, uint32_t* out_k,
                               uint32_t* out_v) {
    std::vector<RunRef> rr;
    for (int r = 0; r < runs; ++r) rr.push_back({rk[r], V ? rv[r] : nullptr, bound[r], off[r], len[r]});
    dc_status st = ensure_scratch(p, V);
    if (st != DC_OK) return st;
    const size_t kb = align_up((size_t)p->n * 4, 256);
    uint32_t* sk = (uint32_t*)p->scratch;
    uint32_t* sv = V ? (uint32_t*)((char*)p->scratch + kb) : nullptr;
    return merge_g<K, V>(p, rr, tmp_k, tmp_v, sk, sv, out_k, out_v);
}

dc_status ensure_mg_state(dc_plan_t p) {
    if (p->mg_state) return DC_OK;
    void* ptr = nullptr;
    if (cudaMalloc(&ptr, 129 * sizeof(unsigned long long)) != cudaSuccess) {
        cudaGetLastError();
        return fail(DC_ERR_OUT_OF_MEMORY, "splitter state cudaMalloc failed");
    }
    p->mg_state = (unsigned long long*)ptr;
    DC_CUDA(p, cudaMemsetAsync(p->mg_state + 128, 0, sizeof(unsigned long long), p->stream));
    return DC_OK;
}


// f4: the D&C sum through the generic O(1)-combine template (dc_reduce.cuh),
// TMA-streamed warp segments of 32 x kSumL elements, one CTA per SM.
constexpr int kSumThreads = 256;
constexpr int kSumL = 68;
constexpr int kSumS = 2;
constexpr size_t kSumSmem = dc::breadth_first_reduce_tma_smem<kSumThreads, kSumL, kSumS>();

dc_status ensure_sum_state(dc_plan_t p) {
    if (p->sum_state) return DC_OK;
    int dev = 0, sms = 148, occ = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    auto* k = dc::breadth_first_reduce_tma<dc::SumI64, kSumThreads, kSumL, kSumS>;
    DC_CUDA(p, cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSumSmem));
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, kSumThreads, kSumSmem);
    const int64_t units = num_tiles(p->n, (int64_t)kSumThreads * kSumL);   // >= 1 segment/warp
    const int64_t grid = (int64_t)sms * (occ > 0 ? occ : 1);
    p->sum_grid = (int)(units < grid ? units : grid);
    void* ptr = nullptr;
    // parts[grid] | ticket (8 B) | result (8 B)
    if (cudaMalloc(&ptr, (size_t)(p->sum_grid + 2) * 8) != cudaSuccess) {
        cudaGetLastError();
        return fail(DC_ERR_OUT_OF_MEMORY, "sum state cudaMalloc failed");
    }
    p->sum_state = (long long*)ptr;
    DC_CUDA(p, cudaMemsetAsync(ptr, 0, (size_t)(p->sum_grid + 2) * 8, p->stream));
    return DC_OK;
}

}  // namespace

namespace dcx {
dc_status fail(dc_status s, const std::string& msg) { return ::fail(s, msg); }
dc_status cuda_fail(dc_plan_t p, cudaError_t e, const char* what) { return ::cuda_fail(p, e, what); }
dc_status local_sort(dc_plan_t p, dc_key_type kt, uint32_t* keys, uint32_t* vals,
                     uint32_t* out_k, uint32_t* out_v) {
    return sort_dispatch(p, kt, keys, vals, out_k, out_v);
}
}  // namespace dcx

// =================================================================== ABI

extern "C" {

const char* dc_version(void) { return "dc-b200 0.1 (sm_100a)"; }

const char* dc_status_string(dc_status s) {
    switch (s) {
        case DC_OK: return "DC_OK";
        case DC_ERR_INVALID_ARG: return "DC_ERR_INVALID_ARG";
        case DC_ERR_UNSUPPORTED: return "DC_ERR_UNSUPPORTED";
        case DC_ERR_OUT_OF_MEMORY: return "DC_ERR_OUT_OF_MEMORY";
        case DC_ERR_CUDA: return "DC_ERR_CUDA";
        case DC_ERR_NCCL: return "DC_ERR_NCCL";
        case DC_ERR_BAD_STATE: return "DC_ERR_BAD_STATE";
    }
    return "DC_ERR_UNKNOWN";
}

const char* dc_last_error(void) { return g_last_error.c_str(); }

dc_status dc_plan(int64_t n, int32_t a, int32_t b, int64_t base_size, dc_plan_t* out) {
    if (!out) return fail(DC_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (n < 1 || n > kMaxN) return fail(DC_ERR_INVALID_ARG, "n must be in [1, 2^31-1]");
    if (a < 2 || b < 2 || a > 1024 || b > 1024)
        return fail(DC_ERR_INVALID_ARG, "a and b must be in [2, 1024]");
    if (base_size < 1 || base_size > n)
        return fail(DC_ERR_INVALID_ARG, "base_size must be in [1, n]");
    dc_plan_s* p = new (std::nothrow) dc_plan_s();
    if (!p) return fail(DC_ERR_OUT_OF_MEMORY, "plan allocation failed");
    p->n = n;
    p->n_global = n;
    p->a = a;
    p->b = b;
    p->base_size = base_size;
    if (const char* e = std::getenv("DC_PIPE_CHUNKS")) p->pipe_chunks = std::atoi(e);  // tuning
    if (const char* e = std::getenv("DC_TWO_LEVEL")) p->two_force = std::atoi(e) != 0;  // tuning
    // Level i: a^i nodes of size ceil(n / b^i); stop at the first level whose
    // size is <= base_size (leaves at level log_b n for base 1).
    int64_t nodes = 1, size = n, bpow = 1;
    for (;;) {
        p->nodes.push_back(nodes);
        p->sizes.push_back(size);
        if (size <= base_size) break;
        if (nodes > INT64_MAX / a) {
            delete p;
            return fail(DC_ERR_INVALID_ARG, "a^L overflows int64");
        }
        nodes *= a;
        bpow = (bpow > INT64_MAX / b) ? INT64_MAX : bpow * b;
        size = (n + bpow - 1) / bpow;
    }
    *out = p;
    return DC_OK;
}

dc_status dc_plan_levels(dc_plan_t p, int32_t* num_levels, int64_t* nodes, int64_t* sizes,
                         int32_t capacity) {
    if (!p || !num_levels) return fail(DC_ERR_INVALID_ARG, "NULL argument");
    *num_levels = (int32_t)p->nodes.size();
    int32_t m = capacity < *num_levels ? capacity : *num_levels;
    for (int32_t i = 0; i < m; ++i) {
        if (nodes) nodes[i] = p->nodes[i];
        if (sizes) sizes[i] = p->sizes[i];
    }
    return DC_OK;
}

dc_status dc_plan_schedule(dc_plan_t p, dc_key_type kt, int32_t with_vals, int32_t* tile,
                           int32_t* fused_levels, int32_t* passes, int32_t* hbm_passes) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (kt != DC_KEY_U32 && kt != DC_KEY_I32 && kt != DC_KEY_F32)
        return fail(DC_ERR_INVALID_ARG, "unknown key type");
    const Decision d = decide(p, kt, with_vals != 0);
    const SortCfg c = cfg_for_runtime(kt, with_vals != 0, d.small);
    const int64_t ft = (int64_t)c.tile() * d.cs;   // fused run width
    if (tile) *tile = (int32_t)ft;
    int f = 0;   // levels of the binary tree inside one fused run: ceil(log2(run))
    while (((int64_t)1 << f) < ft) ++f;
    if (fused_levels) *fused_levels = f;
    const int P = global_passes(p->n, ft);
    if (passes) *passes = P;
    const bool two = d.two && P >= 2;
    if (hbm_passes) *hbm_passes = two ? (P % 2) + (P - P % 2) / 2 : P;
    return DC_OK;
}

dc_status dc_plan_set_two_level(dc_plan_t p, int32_t enable) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (enable < -1 || enable > 1) return fail(DC_ERR_INVALID_ARG, "enable must be -1, 0 or 1");
    p->two_force = enable;
    drop_graphs(p);
    return DC_OK;
}

dc_status dc_plan_set_tile_class(dc_plan_t p, int32_t tile_class) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (tile_class < 0 || tile_class > 2) return fail(DC_ERR_INVALID_ARG, "tile_class must be 0, 1 or 2");
    p->tile_class = tile_class;
    drop_graphs(p);
    return DC_OK;
}

dc_status dc_plan_set_nk1_cluster(dc_plan_t p, int32_t cs) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (!(cs == 0 || cs == 1 || cs == 2 || cs == 4 || cs == 8 || cs == 16))
        return fail(DC_ERR_INVALID_ARG, "cs must be 0, 1, 2, 4, 8 or 16");
    p->nk1_cluster = cs;
    drop_graphs(p);
    return DC_OK;
}

dc_status dc_plan_set_fused_partition(dc_plan_t p, int32_t enable) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    p->fuse_partition = enable != 0;
    drop_graphs(p);
    return DC_OK;
}

dc_status dc_plan_set_pipeline(dc_plan_t p, int32_t chunks) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (chunks < 0 || chunks > 64) return fail(DC_ERR_INVALID_ARG, "chunks must be in [0, 64]");
    p->pipe_chunks = chunks;
    drop_graphs(p);
    return DC_OK;
}

dc_status dc_plan_set_graphs(dc_plan_t p, int32_t enable) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    p->use_graphs = enable != 0;
    drop_graphs(p);
    return DC_OK;
}

dc_status dc_plan_set_stream(dc_plan_t p, void* stream) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    p->stream = (cudaStream_t)stream;
    return DC_OK;
}

dc_status dc_plan_scratch_bytes(dc_plan_t p, int32_t with_vals, size_t* bytes) {
    if (!p || !bytes) return fail(DC_ERR_INVALID_ARG, "NULL argument");
    *bytes = scratch_needed(p->n, with_vals != 0);
    return DC_OK;
}

dc_status dc_plan_set_scratch(dc_plan_t p, void* d, size_t bytes) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (!d || !aligned16(d)) return fail(DC_ERR_INVALID_ARG, "scratch NULL or misaligned");
    if (bytes < scratch_needed(p->n, false))
        return fail(DC_ERR_INVALID_ARG, "scratch smaller than dc_plan_scratch_bytes");
    if (p->scratch && p->own_scratch) cudaFree(p->scratch);
    drop_graphs(p);
    p->scratch = d;
    p->scratch_bytes = bytes;
    p->own_scratch = false;
    return DC_OK;
}

dc_status dc_free(dc_plan_t p) {
    if (!p) return DC_OK;
    if (p->mg) dcx::mg_destroy(p->mg);
    for (auto& t : p->pending) {
        cudaEventDestroy(t.e0);
        cudaEventDestroy(t.e1);
    }
    for (auto e : p->event_pool) cudaEventDestroy(e);
    if (p->scratch && p->own_scratch) cudaFree(p->scratch);
    if (p->ms_tiles) cudaFree(p->ms_tiles);
    if (p->d_stage) cudaFree(p->d_stage);
    for (auto& hs : p->hslot) {
        if (hs.d) cudaFree(hs.d);
        if (hs.in_done) cudaEventDestroy(hs.in_done);
        if (hs.sort_done) cudaEventDestroy(hs.sort_done);
        if (hs.out_done) cudaEventDestroy(hs.out_done);
    }
    if (p->join_in) cudaEventDestroy(p->join_in);
    if (p->join_out) cudaEventDestroy(p->join_out);
    if (p->comp_done) cudaEventDestroy(p->comp_done);
    if (p->h2d) cudaStreamDestroy(p->h2d);
    if (p->d2h) cudaStreamDestroy(p->d2h);
    if (p->comp) cudaStreamDestroy(p->comp);
    if (p->mg_state) cudaFree(p->mg_state);
    if (p->sum_state) cudaFree(p->sum_state);
    for (auto& gc : p->graphs) {
        if (gc.exec) cudaGraphExecDestroy(gc.exec);
        if (gc.graph) cudaGraphDestroy(gc.graph);
    }
    if (p->cap_stream) cudaStreamDestroy(p->cap_stream);
    for (auto st : p->pipe_streams) cudaStreamDestroy(st);
    for (auto ev : p->pipe_events) cudaEventDestroy(ev);
    delete p;
    return DC_OK;
}

int64_t dc_plan_launch_count(dc_plan_t p) { return p ? p->launches : -1; }

dc_status dc_plan_enable_timing(dc_plan_t p, int32_t enable) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    for (auto& t : p->pending) {
        p->event_pool.push_back(t.e0);
        p->event_pool.push_back(t.e1);
    }
    p->pending.clear();
    for (int k = 0; k < DC_KERNEL_COUNT; ++k) {
        p->acc_ms[k] = 0;
        p->acc_n[k] = 0;
    }
    p->timing = enable != 0;
    return DC_OK;
}

dc_status dc_plan_kernel_time(dc_plan_t p, int32_t kernel, double* total_ms, int64_t* launches) {
    if (!p || kernel < 0 || kernel >= DC_KERNEL_COUNT)
        return fail(DC_ERR_INVALID_ARG, "bad plan or kernel id");
    for (auto& t : p->pending) {
        cudaError_t e = cudaEventSynchronize(t.e1);
        if (e != cudaSuccess) return cuda_fail(p, e, "cudaEventSynchronize");
        float ms = 0.f;
        cudaEventElapsedTime(&ms, t.e0, t.e1);
        p->acc_ms[t.kind] += ms;
        p->acc_n[t.kind] += 1;
        p->event_pool.push_back(t.e0);
        p->event_pool.push_back(t.e1);
    }
    p->pending.clear();
    if (total_ms) *total_ms = p->acc_ms[kernel];
    if (launches) *launches = p->acc_n[kernel];
    return DC_OK;
}

static dc_status run_mergesort(dc_plan_t p, dc_key_type kt, void* d_keys, uint32_t* d_vals);

dc_status dc_run_mergesort(dc_plan_t p, dc_key_type kt, void* d_keys, uint32_t* d_vals) {
    const dc_status st = run_mergesort(p, kt, d_keys, d_vals);
    if (st != DC_OK && p && p->mg) dcx::mg_abort(p->mg);   // release the other ranks
    return st;
}

static dc_status run_mergesort(dc_plan_t p, dc_key_type kt, void* d_keys, uint32_t* d_vals) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (p->a != 2 || p->b != 2)
        return fail(DC_ERR_UNSUPPORTED, "runs need a == b == 2");
    if (kt != DC_KEY_U32 && kt != DC_KEY_I32 && kt != DC_KEY_F32)
        return fail(DC_ERR_INVALID_ARG, "unknown key type");
    if (!d_keys || !aligned16(d_keys)) return fail(DC_ERR_INVALID_ARG, "keys NULL or misaligned");
    if (d_vals && !aligned16(d_vals)) return fail(DC_ERR_INVALID_ARG, "vals misaligned");
    if (p->mg) return dcx::mg_sort(p, kt, (uint32_t*)d_keys, d_vals);
    return sort_dispatch(p, kt, (uint32_t*)d_keys, d_vals);
}

dc_status dc_run_mergesort_host(dc_plan_t p, dc_key_type kt, void* h_keys, uint32_t* h_vals) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (p->a != 2 || p->b != 2)
        return fail(DC_ERR_UNSUPPORTED, "runs need a == b == 2");
    if (kt != DC_KEY_U32 && kt != DC_KEY_I32 && kt != DC_KEY_F32)
        return fail(DC_ERR_INVALID_ARG, "unknown key type");
    if (!h_keys) return fail(DC_ERR_INVALID_ARG, "keys NULL");
    if (p->mg) return fail(DC_ERR_UNSUPPORTED, "host-buffer sorts are single-GPU");
    size_t kb = align_up((size_t)p->n * 4, 256);
    st = ensure_stage(p, h_vals ? 2 * kb : kb);
    if (st != DC_OK) return st;
    uint32_t* dk = (uint32_t*)p->d_stage;
    uint32_t* dv = h_vals ? (uint32_t*)((char*)p->d_stage + kb) : nullptr;
    size_t bytes = (size_t)p->n * 4;
    DC_CUDA(p, cudaMemcpyAsync(dk, h_keys, bytes, cudaMemcpyHostToDevice, p->stream));
    if (h_vals) DC_CUDA(p, cudaMemcpyAsync(dv, h_vals, bytes, cudaMemcpyHostToDevice, p->stream));
    st = sort_dispatch(p, kt, dk, dv);
    if (st != DC_OK) return st;
    DC_CUDA(p, cudaMemcpyAsync(h_keys, dk, bytes, cudaMemcpyDeviceToHost, p->stream));
    if (h_vals) DC_CUDA(p, cudaMemcpyAsync(h_vals, dv, bytes, cudaMemcpyDeviceToHost, p->stream));
    DC_CUDA(p, cudaStreamSynchronize(p->stream));
    return DC_OK;
}

dc_status dc_run_maxsubarray_async(dc_plan_t p, const int32_t* d_x, int64_t off,
                                   dc_maxsub_result* d_out) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (p->a != 2 || p->b != 2) return fail(DC_ERR_UNSUPPORTED, "runs need a == b == 2");
    if (!d_x || !aligned16(d_x)) return fail(DC_ERR_INVALID_ARG, "x NULL or misaligned");
    if (!d_out) return fail(DC_ERR_INVALID_ARG, "out NULL");
    return maxsub_launch(p, d_x, off, 0, d_out, nullptr);
}

dc_status dc_run_maxsubarray_tuple_async(dc_plan_t p, const int32_t* d_x, int64_t off,
                                         dc_maxsub_tuple* d_tuple) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (p->a != 2 || p->b != 2) return fail(DC_ERR_UNSUPPORTED, "runs need a == b == 2");
    if (!d_x || !aligned16(d_x)) return fail(DC_ERR_INVALID_ARG, "x NULL or misaligned");
    if (!d_tuple) return fail(DC_ERR_INVALID_ARG, "tuple NULL");
    return maxsub_launch(p, d_x, off, 1, nullptr, d_tuple);
}

dc_status dc_run_maxsubarray(dc_plan_t p, const int32_t* d_x, dc_maxsub_result* h_out) {
    dc_status st = check_plan(p);
    if (st == DC_OK && !h_out) st = fail(DC_ERR_INVALID_ARG, "out NULL");
    if (st == DC_OK && p->mg && (!d_x || !aligned16(d_x)))
        st = fail(DC_ERR_INVALID_ARG, "x NULL or misaligned");
    if (st != DC_OK) {
        if (p && p->mg) dcx::mg_abort(p->mg);
        return st;
    }
    if (p->mg) return dcx::mg_maxsub(p, d_x, h_out);
    st = ensure_ms_state(p);
    if (st != DC_OK) return st;
    st = dc_run_maxsubarray_async(p, d_x, 0, p->ms_res);
    if (st != DC_OK) return st;
    DC_CUDA(p, cudaMemcpyAsync(h_out, p->ms_res, sizeof(dc_maxsub_result),
                               cudaMemcpyDeviceToHost, p->stream));
    DC_CUDA(p, cudaStreamSynchronize(p->stream));
    return DC_OK;
}

dc_status dc_run_maxsubarray_host(dc_plan_t p, const int32_t* h_x, dc_maxsub_result* h_out) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!h_x || !h_out) return fail(DC_ERR_INVALID_ARG, "NULL argument");
    st = ensure_stage(p, align_up((size_t)p->n * 4, 256));
    if (st != DC_OK) return st;
    DC_CUDA(p, cudaMemcpyAsync(p->d_stage, h_x, (size_t)p->n * 4, cudaMemcpyHostToDevice,
                               p->stream));
    return dc_run_maxsubarray(p, (const int32_t*)p->d_stage, h_out);
}

dc_status dc_maxsub_combine_async(dc_plan_t p, const dc_maxsub_tuple* d_tuples, int32_t count,
                                  dc_maxsub_result* d_out) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!d_tuples || !d_out || count < 1) return fail(DC_ERR_INVALID_ARG, "bad arguments");
    dc::nk5_combine_tuples<<<1, 32, 0, p->stream>>>(d_tuples, count, d_out);
    DC_LAUNCHED(p);
    return DC_OK;
}

// ------------------------------------------------ multi-GPU building blocks

int64_t dc_mg_sendbuf_words(int32_t world, int64_t wcap) {
    return world < 2 ? 0 : dc::mg_sendbuf_words(world, wcap);
}

dc_status dc_mg_sample(dc_plan_t p, const uint32_t* d_keys, int64_t n, int64_t stride,
                       uint32_t* d_samples) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!d_keys || !d_samples || n < 1 || stride < 1)
        return fail(DC_ERR_INVALID_ARG, "bad sample arguments");
    const int64_t cnt = (n + stride - 1) / stride;
    dc::mg_sample<<<(unsigned)((cnt + 255) / 256), 256, 0, p->stream>>>(d_keys, stride, cnt,
                                                                       d_samples);
    DC_LAUNCHED(p);
    return DC_OK;
}

dc_status dc_mg_count(dc_plan_t p, dc_key_type kt, const uint32_t* d_keys, int64_t n,
                      int32_t rank, const uint32_t* d_cand, int64_t per_rank, int64_t stride,
                      int64_t cands, int64_t* d_counts) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!d_keys || !d_cand || !d_counts || per_rank < 1 || cands < 1 || cands >= (1LL << 24))
        return fail(DC_ERR_INVALID_ARG, "bad count arguments");
    const unsigned grid = (unsigned)((cands + 255) / 256);
    switch (kt) {
        case DC_KEY_U32:
            dc::mg_count<dc::KeyU32><<<grid, 256, 0, p->stream>>>(d_keys, n, rank, d_cand,
                                                                  per_rank, stride, cands,
                                                                  d_counts);
            break;
        case DC_KEY_I32:
            dc::mg_count<dc::KeyI32><<<grid, 256, 0, p->stream>>>(d_keys, n, rank, d_cand,
                                                                  per_rank, stride, cands,
                                                                  d_counts);
            break;
        case DC_KEY_F32:
            dc::mg_count<dc::KeyF32><<<grid, 256, 0, p->stream>>>(d_keys, n, rank, d_cand,
                                                                  per_rank, stride, cands,
                                                                  d_counts);
            break;
        default:
            return fail(DC_ERR_INVALID_ARG, "unknown key type");
    }
    DC_LAUNCHED(p);
    return DC_OK;
}

dc_status dc_mg_windows(dc_plan_t p, const uint32_t* d_keys, int64_t n, int32_t rank,
                        int32_t world, const int64_t* d_counts, const int64_t* d_ranks,
                        int64_t per_rank, int64_t cands, int64_t wcap, uint32_t* d_sendbuf) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!d_keys || !d_counts || !d_ranks || !d_sendbuf || world < 2 || world > 64 ||
        rank < 0 || rank >= world || cands < 1 || cands >= (1LL << 24))
        return fail(DC_ERR_INVALID_ARG, "bad window arguments");
    st = ensure_mg_state(p);
    if (st != DC_OK) return st;
    unsigned long long* lo = p->mg_state;
    unsigned long long* hi = p->mg_state + 64;
    DC_CUDA(p, cudaMemsetAsync(lo, 0x00, 64 * sizeof(unsigned long long), p->stream));
    DC_CUDA(p, cudaMemsetAsync(hi, 0xFF, 64 * sizeof(unsigned long long), p->stream));
    dc::mg_brackets<<<(unsigned)((cands + 255) / 256), 256, 0, p->stream>>>(d_ranks, cands, world,
                                                                          n, lo, hi);
    DC_LAUNCHED(p);
    dc::mg_windows<<<world - 1, 256, 0, p->stream>>>(d_keys, n, rank, world, n, d_counts, d_ranks,
                                                      per_rank, wcap, lo, hi, d_sendbuf,
                                                      (int*)(p->mg_state + 128));
    DC_LAUNCHED(p);
    return DC_OK;
}

dc_status dc_mg_split_matrix(dc_plan_t p, dc_key_type kt, const uint32_t* d_gathered,
                             int32_t world, int64_t shard_n, int64_t wcap, int64_t* d_cmat) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!d_gathered || !d_cmat || world < 2 || world > 64 || wcap < 1)
        return fail(DC_ERR_INVALID_ARG, "bad split-matrix arguments");
    const size_t smem = (size_t)world * wcap * 4;
    if (smem > 200 * 1024) return fail(DC_ERR_INVALID_ARG, "world * wcap too large");
    switch (kt) {
        case DC_KEY_U32: {
            auto* k = dc::mg_split_matrix<dc::KeyU32>;
            DC_CUDA(p, cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                            (int)smem));
            k<<<world - 1, 256, smem, p->stream>>>(d_gathered, world, shard_n, wcap, d_cmat);
            break;
        }
        case DC_KEY_I32: {
            auto* k = dc::mg_split_matrix<dc::KeyI32>;
            DC_CUDA(p, cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                            (int)smem));
            k<<<world - 1, 256, smem, p->stream>>>(d_gathered, world, shard_n, wcap, d_cmat);
            break;
        }
        case DC_KEY_F32: {
            auto* k = dc::mg_split_matrix<dc::KeyF32>;
            DC_CUDA(p, cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                            (int)smem));
            k<<<world - 1, 256, smem, p->stream>>>(d_gathered, world, shard_n, wcap, d_cmat);
            break;
        }
        default:
            return fail(DC_ERR_INVALID_ARG, "unknown key type");
    }
    DC_LAUNCHED(p);
    return DC_OK;
}

dc_status dc_mg_error(dc_plan_t p, int32_t* h_err) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!h_err) return fail(DC_ERR_INVALID_ARG, "NULL argument");
    *h_err = 0;
    if (!p->mg_state) return DC_OK;
    int v = 0;
    DC_CUDA(p, cudaMemcpyAsync(&v, p->mg_state + 128, sizeof(int), cudaMemcpyDeviceToHost,
                               p->stream));
    DC_CUDA(p, cudaStreamSynchronize(p->stream));
    *h_err = v;
    return DC_OK;
}

dc_status dc_mg_merge_runs(dc_plan_t p, dc_key_type kt, uint32_t* d_in_keys, uint32_t* d_in_vals,
                           uint32_t* d_out_keys, uint32_t* d_out_vals, const int64_t* h_run_len,
                           int32_t runs) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!d_in_keys || !d_out_keys || !h_run_len || runs < 1 ||
        (d_in_vals == nullptr) != (d_out_vals == nullptr))
        return fail(DC_ERR_INVALID_ARG, "bad merge arguments");
    if (!aligned16(d_in_keys) || !aligned16(d_out_keys) ||
        (d_in_vals && (!aligned16(d_in_vals) || !aligned16(d_out_vals))))
        return fail(DC_ERR_INVALID_ARG, "buffers must be 16-byte aligned");
    std::vector<int64_t> lens(h_run_len, h_run_len + runs);
    for (int64_t l : lens)
        if (l < 0) return fail(DC_ERR_INVALID_ARG, "negative run length");
    const bool v = d_in_vals != nullptr;
    switch (kt) {
        case DC_KEY_U32:
            return v ? mg_merge_typed<dc::KeyU32, true>(p, d_in_keys, d_in_vals, d_out_keys,
                                                        d_out_vals, lens)
                     : mg_merge_typed<dc::KeyU32, false>(p, d_in_keys, nullptr, d_out_keys,
                                                         nullptr, lens);
        case DC_KEY_I32:
            return v ? mg_merge_typed<dc::KeyI32, true>(p, d_in_keys, d_in_vals, d_out_keys,
                                                        d_out_vals, lens)
                     : mg_merge_typed<dc::KeyI32, false>(p, d_in_keys, nullptr, d_out_keys,
                                                         nullptr, lens);
        case DC_KEY_F32:
            return v ? mg_merge_typed<dc::KeyF32, true>(p, d_in_keys, d_in_vals, d_out_keys,
                                                        d_out_vals, lens)
                     : mg_merge_typed<dc::KeyF32, false>(p, d_in_keys, nullptr, d_out_keys,
                                                         nullptr, lens);
    }
    return fail(DC_ERR_INVALID_ARG, "unknown key type");
}

dc_status dc_mg_merge_peers(dc_plan_t p, dc_key_type kt, const uint32_t* const* h_run_keys,
                            const uint32_t* const* h_run_vals, const int64_t* h_bound,
                            const int64_t* h_off, const int64_t* h_len, int32_t runs,
                            uint32_t* d_tmp_keys, uint32_t* d_tmp_vals, uint32_t* d_out_keys,
                            uint32_t* d_out_vals) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    const bool v = d_out_vals != nullptr;
    if (!h_run_keys || !h_bound || !h_off || !h_len || runs < 1 || !d_out_keys ||
        (v && !h_run_vals) || (runs > 4 && (!d_tmp_keys || (v && !d_tmp_vals))))
        return fail(DC_ERR_INVALID_ARG, "bad peer-merge arguments");
    for (int r = 0; r < runs; ++r) {
        if (!h_run_keys[r] || !aligned16(h_run_keys[r]) ||
            (v && (!h_run_vals[r] || !aligned16(h_run_vals[r]))))
            return fail(DC_ERR_INVALID_ARG, "run buffers must be 16-byte aligned");
        if (h_off[r] < 0 || h_len[r] < 0 || h_off[r] + h_len[r] > h_bound[r])
            return fail(DC_ERR_INVALID_ARG, "run outside its buffer");
    }
    if (!aligned16(d_out_keys) || (v && !aligned16(d_out_vals)) ||
        (d_tmp_keys && !aligned16(d_tmp_keys)) || (d_tmp_vals && !aligned16(d_tmp_vals)))
        return fail(DC_ERR_INVALID_ARG, "buffers must be 16-byte aligned");
#define DC_PEERS(KT)                                                                         \
    return v ? mg_merge_peers_typed<KT, true>(p, h_run_keys, h_run_vals, h_bound, h_off, h_len, \
                                              runs, d_tmp_keys, d_tmp_vals, d_out_keys,       \
                                              d_out_vals)                                     \
             : mg_merge_peers_typed<KT, false>(p, h_run_keys, nullptr, h_bound, h_off, h_len,  \
                                               runs, d_tmp_keys, nullptr, d_out_keys, nullptr)
    switch (kt) {
        case DC_KEY_U32: DC_PEERS(dc::KeyU32);
        case DC_KEY_I32: DC_PEERS(dc::KeyI32);
        case DC_KEY_F32: DC_PEERS(dc::KeyF32);
    }
#undef DC_PEERS
    return fail(DC_ERR_INVALID_ARG, "unknown key type");
}

// --------------------------------------------------- D&C sum

dc_status dc_run_sum_async(dc_plan_t p, const int32_t* d_x, int64_t* d_out) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (p->a != 2 || p->b != 2) return fail(DC_ERR_UNSUPPORTED, "runs need a == b == 2");
    if (!d_x || !d_out) return fail(DC_ERR_INVALID_ARG, "NULL argument");
    st = ensure_sum_state(p);
    if (st != DC_OK) return st;
    if (!aligned16(d_x)) return fail(DC_ERR_INVALID_ARG, "x must be 16-byte aligned");
    dc::breadth_first_reduce_tma<dc::SumI64, kSumThreads, kSumL, kSumS>
        <<<p->sum_grid, kSumThreads, kSumSmem, p->stream>>>(
            d_x, p->n, dc::breadth_first_reduce_tma_rw<kSumThreads, kSumL>(p->n, p->sum_grid),
            p->sum_state, (unsigned int*)(p->sum_state + p->sum_grid), (long long*)d_out);
    DC_LAUNCHED(p);
    return DC_OK;
}

dc_status dc_run_sum(dc_plan_t p, const int32_t* d_x, int64_t* h_out) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!h_out) return fail(DC_ERR_INVALID_ARG, "NULL argument");
    st = ensure_sum_state(p);
    if (st != DC_OK) return st;
    long long* d_res = p->sum_state + p->sum_grid + 1;
    st = dc_run_sum_async(p, d_x, (int64_t*)d_res);
    if (st != DC_OK) return st;
    DC_CUDA(p, cudaMemcpyAsync(h_out, d_res, 8, cudaMemcpyDeviceToHost, p->stream));
    DC_CUDA(p, cudaStreamSynchronize(p->stream));
    return DC_OK;
}

dc_status dc_run_sum_alg5(dc_plan_t p, int64_t* d_work, int64_t* h_out) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!d_work || !h_out) return fail(DC_ERR_INVALID_ARG, "NULL argument");
    for (long long len = p->n; len > 1;) {          // one launch per level (Alg 5)
        const long long m = (len + 1) / 2;
        dc::alg5_sum_level<<<(unsigned)((m + 255) / 256), 256, 0, p->stream>>>(
            (long long*)d_work, len, m);
        DC_LAUNCHED(p);
        len = m;
    }
    DC_CUDA(p, cudaMemcpyAsync(h_out, d_work, 8, cudaMemcpyDeviceToHost, p->stream));
    DC_CUDA(p, cudaStreamSynchronize(p->stream));
    return DC_OK;
}

// ------------------------------------------- streaming end-to-end sorts

dc_status dc_sort_host_submit(dc_plan_t p, dc_key_type kt, const void* h_in_keys,
                              const uint32_t* h_in_vals, void* h_out_keys, uint32_t* h_out_vals) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (p->a != 2 || p->b != 2) return fail(DC_ERR_UNSUPPORTED, "runs need a == b == 2");
    if (kt != DC_KEY_U32 && kt != DC_KEY_I32 && kt != DC_KEY_F32)
        return fail(DC_ERR_INVALID_ARG, "unknown key type");
    if (!h_in_keys || !h_out_keys || (h_in_vals == nullptr) != (h_out_vals == nullptr))
        return fail(DC_ERR_INVALID_ARG, "bad host buffers");
    if (p->mg) return fail(DC_ERR_UNSUPPORTED, "host-buffer sorts are single-GPU");
    if (!p->h2d) {
        DC_CUDA(p, cudaStreamCreateWithFlags(&p->h2d, cudaStreamNonBlocking));
        DC_CUDA(p, cudaStreamCreateWithFlags(&p->d2h, cudaStreamNonBlocking));
        DC_CUDA(p, cudaStreamCreateWithFlags(&p->comp, cudaStreamNonBlocking));
        DC_CUDA(p, cudaEventCreateWithFlags(&p->join_in, cudaEventDisableTiming));
        DC_CUDA(p, cudaEventCreateWithFlags(&p->join_out, cudaEventDisableTiming));
        DC_CUDA(p, cudaEventCreateWithFlags(&p->comp_done, cudaEventDisableTiming));
        for (auto& hs : p->hslot) {
            DC_CUDA(p, cudaEventCreateWithFlags(&hs.in_done, cudaEventDisableTiming));
            DC_CUDA(p, cudaEventCreateWithFlags(&hs.sort_done, cudaEventDisableTiming));
            DC_CUDA(p, cudaEventCreateWithFlags(&hs.out_done, cudaEventDisableTiming));
            DC_CUDA(p, cudaEventRecord(hs.out_done, p->d2h));
        }
    }
    auto& hs = p->hslot[p->submits % dc_plan_s::kHostSlots];
    const size_t kb = align_up((size_t)p->n * 4, 256);
    const size_t need = h_in_vals ? 2 * kb : kb;
    if (hs.bytes < need) {
        DC_CUDA(p, cudaEventSynchronize(hs.out_done));
        drop_graphs(p);
        if (hs.d) cudaFree(hs.d);
        hs.d = nullptr;
        if (cudaMalloc(&hs.d, need) != cudaSuccess) {
            cudaGetLastError();
            hs.bytes = 0;
            return fail(DC_ERR_OUT_OF_MEMORY, "host-sort slot cudaMalloc failed");
        }
        hs.bytes = need;
    }
    uint32_t* dk = (uint32_t*)hs.d;
    uint32_t* dv = h_in_vals ? (uint32_t*)((char*)hs.d + kb) : nullptr;
    const size_t bytes = (size_t)p->n * 4;
    // copy in after the work already queued on the plan stream, and once the
    // slot's previous result has left
    DC_CUDA(p, cudaEventRecord(p->join_in, p->stream));
    DC_CUDA(p, cudaStreamWaitEvent(p->h2d, p->join_in, 0));
    DC_CUDA(p, cudaStreamWaitEvent(p->h2d, hs.out_done, 0));
    DC_CUDA(p, cudaMemcpyAsync(dk, h_in_keys, bytes, cudaMemcpyHostToDevice, p->h2d));
    if (dv) DC_CUDA(p, cudaMemcpyAsync(dv, h_in_vals, bytes, cudaMemcpyHostToDevice, p->h2d));
    DC_CUDA(p, cudaEventRecord(hs.in_done, p->h2d));
    // sort on the compute stream (sorts of the slots serialise: shared scratch)
    DC_CUDA(p, cudaStreamWaitEvent(p->comp, hs.in_done, 0));
    cudaStream_t user = p->stream;
    p->stream = p->comp;
    st = sort_dispatch(p, kt, dk, dv);
    p->stream = user;
    if (st != DC_OK) return st;
    DC_CUDA(p, cudaEventRecord(hs.sort_done, p->comp));
    DC_CUDA(p, cudaEventRecord(p->comp_done, p->comp));
    // copy out
    DC_CUDA(p, cudaStreamWaitEvent(p->d2h, hs.sort_done, 0));
    DC_CUDA(p, cudaMemcpyAsync(h_out_keys, dk, bytes, cudaMemcpyDeviceToHost, p->d2h));
    if (dv) DC_CUDA(p, cudaMemcpyAsync(h_out_vals, dv, bytes, cudaMemcpyDeviceToHost, p->d2h));
    DC_CUDA(p, cudaEventRecord(hs.out_done, p->d2h));
    p->submits++;
    return DC_OK;
}

dc_status dc_sort_host_wait(dc_plan_t p) {
    dc_status st = check_plan(p);
    if (st != DC_OK) return st;
    if (!p->d2h) return DC_OK;
    DC_CUDA(p, cudaEventRecord(p->join_out, p->d2h));
    DC_CUDA(p, cudaStreamWaitEvent(p->stream, p->join_out, 0));   // the plan stream joins
    DC_CUDA(p, cudaStreamSynchronize(p->d2h));
    return DC_OK;
}

}  // extern "C"
