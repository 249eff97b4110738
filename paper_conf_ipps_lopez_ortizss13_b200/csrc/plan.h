// plan.h -- the plan object shared by the library's translation units
// (internal; the ABI sees only the opaque dc_plan_t of include/dc.h).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <vector>

#include "dc.h"

namespace dcx {
struct MgCtx;   // multi-GPU runtime state (mg_runtime.cu)

// Internal entry points shared between dc_api.cu and mg_runtime.cu.
dc_status fail(dc_status s, const std::string& msg);                 // sets dc_last_error
dc_status cuda_fail(dc_plan_t p, cudaError_t e, const char* what);   // poisons the plan
// sorts keys (+vals) into out_k (+out_v); nullptr outputs = in place
dc_status local_sort(dc_plan_t p, dc_key_type kt, uint32_t* keys, uint32_t* vals,
                     uint32_t* out_k = nullptr, uint32_t* out_v = nullptr);
dc_status mg_sort(dc_plan_t p, dc_key_type kt, uint32_t* keys, uint32_t* vals);
dc_status mg_maxsub(dc_plan_t p, const int32_t* x, dc_maxsub_result* h_out);
void mg_destroy(MgCtx* c);
void mg_abort(MgCtx* c);   // a failing member releases the other ranks (loopback)
}  // namespace dcx

struct dc_plan_s {
    int64_t n = 0;
    int32_t a = 2, b = 2;
    int64_t base_size = 1;
    std::vector<int64_t> nodes, sizes;
    cudaStream_t stream = nullptr;
    bool bad = false;
    int64_t launches = 0;
    // scratch (keys ping-pong, values ping-pong, partition array)
    void* scratch = nullptr;
    size_t scratch_bytes = 0;
    bool own_scratch = false;
    // max-subarray state
    dc_maxsub_tuple* ms_tiles = nullptr;
    unsigned int* ms_ticket = nullptr;
    dc_maxsub_result* ms_res = nullptr;
    CUtensorMap ms_map;                // 2-D row view of the last max-subarray input
    const void* ms_map_x = nullptr;
    int64_t ms_map_n = -1, ms_map_w = 0;
    // CUDA graphs of the sort's launch sequence, per (keys, vals, key type)
    struct GraphCache {
        uint32_t* keys;
        uint32_t* vals;
        uint32_t* out;
        dc_key_type kt;
        cudaGraph_t graph;
        cudaGraphExec_t exec;
        int64_t launches;
    };
    bool use_graphs = true;
    std::vector<GraphCache> graphs;
    cudaStream_t cap_stream = nullptr;
    // chunked pipeline: chunk c's fused bottom levels and in-chunk merge levels
    // run on their own stream, so one chunk's HBM-bound merges could overlap
    // the next chunk's compute-bound NK1; the top levels follow on the plan
    // stream.  Off by default: measured slower at 2^28 (2/8/16 chunks: 7.51 /
    // 7.12 / 6.79 ms vs 6.57) -- NK1 fills an SM's registers and shared memory,
    // so the kernels split SMs instead of sharing them and NK3 loses bandwidth.
    int pipe_chunks = 1;
    std::vector<cudaStream_t> pipe_streams;
    std::vector<cudaEvent_t> pipe_events;   // [0] fork, [1..] per-chunk joins
    // two levels of the merge tree per HBM pass for keys-only sorts (f1).
    // Off by default: bit-exact, and its 4-way tile merge beats two one-level
    // passes (0.545 vs 0.626 ms per two levels at 2^28), but the exact
    // two-level partition costs 0.21 ms per pass vs 2 x 0.03.
    // Schedule of the sort (the planner, model.cu, picks the tile
    // class and the pass kind per (n, key type, values) unless overridden)
    int two_force = -1;       // -1 planner; 0 one level per HBM pass; 1 two levels (4-way)
    int tile_class = 0;       // 0 planner; 1 quarter-size tiles; 2 full tiles
    bool fuse_partition = true;   // small sorts: merge CTAs find their own co-ranks
    // NK1 cluster size for keys-only u32/i32 sorts (f2: log2(CS) more levels on
    // chip through distributed shared memory): 0 the planner's rule, 1 off,
    // 2/4/8/16 forced
    int nk1_cluster = 0;
    // D&C sum (f4): per-CTA parts + ticket + result
    long long* sum_state = nullptr;
    int sum_grid = 0;
    // multi-GPU splitter state: bracket packs [64] lo, [64] hi, error flag
    unsigned long long* mg_state = nullptr;
    // host-buffer (end-to-end) staging
    void* d_stage = nullptr;
    size_t d_stage_bytes = 0;
    // streaming host sorts: three device slots (copy-in of step i+2 overlaps the
    // copy-out of step i and the sort of step i+1), copy-in / compute / copy-out streams
    struct HostSlot {
        void* d = nullptr;              // keys [n] (+ vals [n])
        size_t bytes = 0;
        cudaEvent_t in_done = nullptr, sort_done = nullptr, out_done = nullptr;
    };
    static constexpr int kHostSlots = 3;
    HostSlot hslot[kHostSlots];
    cudaStream_t h2d = nullptr, d2h = nullptr, comp = nullptr;
    cudaEvent_t join_in = nullptr, join_out = nullptr;   // order against the plan stream
    cudaEvent_t comp_done = nullptr;   // last host-slot sort on comp (scratch users wait on it)
    int64_t submits = 0;
    // library-owned communicator (dc_plan_set_comm / dc_plan_set_loopback):
    // n above is then this rank's shard, n_global the whole problem
    dcx::MgCtx* mg = nullptr;
    int64_t n_global = 0;
    int64_t mg_stride = 4096;   // splitter sample stride S
    bool mg_p2p = false;        // fused exchange (peer reads); NCCL all-to-all until measured across GPUs
    // per-kernel CUDA-event timing (instrumentation, off by default)
    bool timing = false;
    struct Timed { int kind; cudaEvent_t e0, e1; };
    std::vector<Timed> pending;
    std::vector<cudaEvent_t> event_pool;
    double acc_ms[DC_KERNEL_COUNT] = {0};
    int64_t acc_n[DC_KERNEL_COUNT] = {0};
};
