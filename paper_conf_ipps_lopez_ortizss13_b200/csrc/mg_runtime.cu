// mg_runtime.cu -- the library-owned multi-GPU runtime (b).
//
// dc_plan_set_comm binds a plan to an NCCL communicator (dc_plan_set_loopback
// to an in-process group of threads sharing one GPU, for tests); after that,
// dc_run_mergesort / dc_run_maxsubarray on a plan of GLOBAL size n take this
// rank's shard of m = n/world elements and run the whole distributed method:
//
//   levels >= log2 G : the single-GPU breadth-first sort of the shard
//                      (independent subproblems, no communication);
//   top log2 G levels: ONE exchange (the paper's single-transfer principle,
//                      P:L474-478, applied between GPUs):
//     a7  samples -> all-gather -> composite counts -> all-reduce ->
//         bracketing windows -> all-gather -> exact split matrix (kernels of
//         mg_kernels.cuh, collectives here), one host sync for the sizes;
//     a8  all-to-all of the key (+ value) ranges (NCCL send/recv group);
//     a9  local stable G-way merge of the received runs.
//   a10 max-subarray: per-rank summary tuple -> all-gather -> ordered combine.
//
// The collectives sit behind a four-call interface (Coll): NcclColl (NCCL is
// dlopen'ed, so the library reuses the copy torch already loaded and has no
// link-time NCCL dependency) and LoopColl (device-to-device copies between the
// buffers of G threads, ordered with events, host barriers between phases).
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <chrono>
#include <condition_variable>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <type_traits>
#include <vector>

#include "dc.h"
#include "plan.h"

static_assert(NCCL_UNIQUE_ID_BYTES == 128, "dc_get_unique_id carries 128 bytes");
static_assert(sizeof(dc_maxsub_tuple) % 8 == 0, "tuples travel as bytes");

// ------------------------------------------------------------ loopback group

struct dc_loopback_s {
    int world = 0;
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    uint64_t gen = 0;
    bool aborted = false;
    std::vector<bool> joined;
    // per-rank publications, valid between a collective's two barriers
    std::vector<const void*> ptr;
    std::vector<const uint32_t* const*> bufs;
    std::vector<const int64_t*> scnt, soff;
    std::vector<cudaEvent_t> ready, done;
};

namespace dcx {
namespace {

// --------------------------------------------------------------- NCCL loader

struct NcclApi {
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t,
                              ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t,
                         cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
    std::string error;   // empty when loaded
};

const NcclApi& nccl() {
    static const NcclApi api = [] {
        NcclApi a;
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);   // torch's copy, if loaded
        if (!h)
            if (const char* e = std::getenv("DC_NCCL_LIB")) h = dlopen(e, RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            const char* why = dlerror();
            a.error = std::string("cannot load libnccl.so.2: ") + (why ? why : "?");
            return a;
        }
        bool all = true;
        auto sym = [&](auto& f, const char* name) {
            f = reinterpret_cast<std::remove_reference_t<decltype(f)>>(dlsym(h, name));
            all = all && f != nullptr;
        };
        sym(a.GetUniqueId, "ncclGetUniqueId");
        sym(a.CommInitRank, "ncclCommInitRank");
        sym(a.CommDestroy, "ncclCommDestroy");
        sym(a.AllGather, "ncclAllGather");
        sym(a.AllReduce, "ncclAllReduce");
        sym(a.Send, "ncclSend");
        sym(a.Recv, "ncclRecv");
        sym(a.GroupStart, "ncclGroupStart");
        sym(a.GroupEnd, "ncclGroupEnd");
        sym(a.GetErrorString, "ncclGetErrorString");
        if (!all) a.error = "libnccl.so.2 lacks a required symbol";
        return a;
    }();
    return api;
}

dc_status nccl_check(ncclResult_t r, const char* what) {
    if (r == ncclSuccess) return DC_OK;
    return fail(DC_ERR_NCCL, std::string(what) + ": " + nccl().GetErrorString(r));
}

dc_status cu_check(cudaError_t e, const char* what) {
    if (e == cudaSuccess) return DC_OK;
    return fail(DC_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

#define MG_TRY(x)                            \
    do {                                     \
        dc_status s_ = (x);                  \
        if (s_ != DC_OK) return s_;          \
    } while (0)
#define MG_CU(x) MG_TRY(cu_check((x), #x))

// ------------------------------------------------------- collective backends

struct Coll {
    int rank = 0, world = 1;
    virtual ~Coll() = default;
    // recv[r*bytes, (r+1)*bytes) = rank r's send, for every r
    virtual dc_status all_gather(const void* send, void* recv, size_t bytes, cudaStream_t s) = 0;
    virtual dc_status all_reduce_sum_i64(int64_t* buf, size_t count, cudaStream_t s) = 0;
    // nbuf parallel buffers of 4-byte elements: elements [soff[d], soff[d]+scnt[d])
    // of send[b] go to rank d; rank q's piece lands at recv[b] + roff[q] (rcnt[q]).
    virtual dc_status all_to_allv(int nbuf, const uint32_t* const* send, uint32_t* const* recv,
                                  const int64_t* scnt, const int64_t* soff, const int64_t* rcnt,
                                  const int64_t* roff, cudaStream_t s) = 0;
    virtual void abort() {}
    // Stream-ordered barrier: work after it on any rank's stream follows every
    // rank's work before it.
    virtual dc_status barrier(cudaStream_t s) = 0;
    // Peer access: every rank's `mine` (a cudaMalloc base) mapped into this
    // process (peers[rank] = mine); *ok = 0 if this rank cannot map them all.
    virtual dc_status share_buffer(void* mine, std::vector<void*>& peers, int* ok,
                                   cudaStream_t s) = 0;
    virtual void unshare(std::vector<void*>& peers) { (void)peers; }
};

struct NcclColl final : Coll {
    ncclComm_t comm = nullptr;
    char* stage = nullptr;   // device staging for barrier words and IPC handles
    ~NcclColl() override {
        if (comm) nccl().CommDestroy(comm);
        if (stage) cudaFree(stage);
    }
    dc_status ensure_stage() {
        if (!stage) MG_CU(cudaMalloc(&stage, 256 + (size_t)(world + 1) * 64));
        return DC_OK;
    }
    dc_status barrier(cudaStream_t s) override {
        MG_TRY(ensure_stage());
        return nccl_check(nccl().AllReduce(stage, stage, 1, ncclInt64, ncclSum, comm, s),
                          "ncclAllReduce(barrier)");
    }
    // CUDA IPC over the node's NVLink/NVSwitch fabric: all-gather the 64-byte
    // handles, open every peer's (lazy peer access).
    dc_status share_buffer(void* mine, std::vector<void*>& peers, int* ok,
                           cudaStream_t s) override {
        MG_TRY(ensure_stage());
        peers.assign(world, nullptr);
        peers[rank] = mine;
        *ok = 1;
        cudaIpcMemHandle_t h;
        std::memset(&h, 0, sizeof h);
        if (!mine || cudaIpcGetMemHandle(&h, mine) != cudaSuccess) {
            cudaGetLastError();
            *ok = 0;
        }
        static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
        char* mine_d = stage + 256;
        char* all_d = stage + 256 + 64;
        MG_CU(cudaMemcpyAsync(mine_d, &h, 64, cudaMemcpyHostToDevice, s));
        MG_TRY(all_gather(mine_d, all_d, 64, s));
        std::vector<cudaIpcMemHandle_t> hs(world);
        MG_CU(cudaMemcpyAsync(hs.data(), all_d, (size_t)world * 64, cudaMemcpyDeviceToHost, s));
        MG_CU(cudaStreamSynchronize(s));
        for (int q = 0; q < world && *ok; ++q) {
            if (q == rank) continue;
            void* ptr = nullptr;
            if (cudaIpcOpenMemHandle(&ptr, hs[q], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
                cudaGetLastError();
                *ok = 0;
                break;
            }
            peers[q] = ptr;
        }
        return DC_OK;
    }
    void unshare(std::vector<void*>& peers) override {
        for (int q = 0; q < (int)peers.size(); ++q)
            if (q != rank && peers[q]) cudaIpcCloseMemHandle(peers[q]);
        peers.clear();
    }
    dc_status all_gather(const void* send, void* recv, size_t bytes, cudaStream_t s) override {
        return nccl_check(nccl().AllGather(send, recv, bytes, ncclUint8, comm, s), "ncclAllGather");
    }
    dc_status all_reduce_sum_i64(int64_t* buf, size_t count, cudaStream_t s) override {
        return nccl_check(nccl().AllReduce(buf, buf, count, ncclInt64, ncclSum, comm, s),
                          "ncclAllReduce");
    }
    dc_status all_to_allv(int nbuf, const uint32_t* const* send, uint32_t* const* recv,
                          const int64_t* scnt, const int64_t* soff, const int64_t* rcnt,
                          const int64_t* roff, cudaStream_t s) override {
        const NcclApi& n = nccl();
        dc_status st = nccl_check(n.GroupStart(), "ncclGroupStart");
        if (st != DC_OK) return st;
        for (int b = 0; b < nbuf && st == DC_OK; ++b)
            for (int d = 0; d < world && st == DC_OK; ++d) {
                if (scnt[d] > 0)
                    st = nccl_check(n.Send(send[b] + soff[d], (size_t)scnt[d], ncclUint32, d, comm, s),
                                    "ncclSend");
                if (st == DC_OK && rcnt[d] > 0)
                    st = nccl_check(n.Recv(recv[b] + roff[d], (size_t)rcnt[d], ncclUint32, d, comm, s),
                                    "ncclRecv");
            }
        const dc_status st2 = nccl_check(n.GroupEnd(), "ncclGroupEnd");
        return st != DC_OK ? st : st2;
    }
};

dc_status lb_barrier(dc_loopback_s* g) {
    std::unique_lock<std::mutex> lk(g->mu);
    if (g->aborted) return fail(DC_ERR_NCCL, "loopback group aborted by a member");
    const uint64_t my = g->gen;
    if (++g->arrived == g->world) {
        g->arrived = 0;
        ++g->gen;
        g->cv.notify_all();
        return DC_OK;
    }
    const bool woke = g->cv.wait_for(lk, std::chrono::seconds(120),
                                     [&] { return g->gen != my || g->aborted; });
    if (!woke) {
        g->aborted = true;
        g->cv.notify_all();
        return fail(DC_ERR_NCCL, "loopback barrier timed out");
    }
    if (g->gen == my) return fail(DC_ERR_NCCL, "loopback group aborted by a member");
    return DC_OK;
}

__global__ void sum_rows_i64(const int64_t* __restrict__ rows, int world, int64_t count,
                             int64_t* __restrict__ out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
         i += (int64_t)gridDim.x * blockDim.x) {
        int64_t acc = 0;
        for (int r = 0; r < world; ++r) acc += rows[r * count + i];
        out[i] = acc;
    }
}

struct LoopColl final : Coll {
    dc_loopback_s* g = nullptr;
    int64_t* tmp = nullptr;   // all-reduce gather space (world x count)
    size_t tmp_bytes = 0;
    ~LoopColl() override {
        if (tmp) cudaFree(tmp);
        if (g) {
            std::lock_guard<std::mutex> lk(g->mu);
            g->joined[rank] = false;
        }
    }
    void abort() override {
        std::lock_guard<std::mutex> lk(g->mu);
        g->aborted = true;
        g->cv.notify_all();
    }
    dc_status barrier(cudaStream_t s) override {
        MG_CU(cudaEventRecord(g->ready[rank], s));
        MG_TRY(lb_barrier(g));
        for (int r = 0; r < world; ++r) MG_CU(cudaStreamWaitEvent(s, g->ready[r], 0));
        return lb_barrier(g);
    }
    // One process, one device: the peers' buffers are directly addressable.
    dc_status share_buffer(void* mine, std::vector<void*>& peers, int* ok,
                           cudaStream_t s) override {
        (void)s;
        g->ptr[rank] = mine;
        MG_TRY(lb_barrier(g));
        peers.resize(world);
        for (int r = 0; r < world; ++r) peers[r] = const_cast<void*>(g->ptr[r]);
        *ok = 1;
        return lb_barrier(g);
    }
    // Second half of every collective: signal that this rank's reads are
    // enqueued, and order this stream after every rank's reads of our buffers.
    dc_status finish(cudaStream_t s) {
        MG_CU(cudaEventRecord(g->done[rank], s));
        MG_TRY(lb_barrier(g));
        for (int r = 0; r < world; ++r) MG_CU(cudaStreamWaitEvent(s, g->done[r], 0));
        return DC_OK;
    }
    dc_status all_gather(const void* send, void* recv, size_t bytes, cudaStream_t s) override {
        g->ptr[rank] = send;
        MG_CU(cudaEventRecord(g->ready[rank], s));
        MG_TRY(lb_barrier(g));
        for (int r = 0; r < world; ++r) {
            MG_CU(cudaStreamWaitEvent(s, g->ready[r], 0));
            if (bytes)
                MG_CU(cudaMemcpyAsync((char*)recv + r * bytes, g->ptr[r], bytes,
                                      cudaMemcpyDeviceToDevice, s));
        }
        return finish(s);
    }
    dc_status all_reduce_sum_i64(int64_t* buf, size_t count, cudaStream_t s) override {
        const size_t need = (size_t)world * count * sizeof(int64_t);
        if (tmp_bytes < need) {
            if (tmp) cudaFree(tmp);
            tmp = nullptr;
            tmp_bytes = 0;
            MG_CU(cudaMalloc(&tmp, need));
            tmp_bytes = need;
        }
        MG_TRY(all_gather(buf, tmp, count * sizeof(int64_t), s));
        if (count) {
            const int grid = (int)std::min<int64_t>(1024, ((int64_t)count + 255) / 256);
            sum_rows_i64<<<grid, 256, 0, s>>>(tmp, world, (int64_t)count, buf);
            MG_CU(cudaGetLastError());
        }
        return DC_OK;
    }
    dc_status all_to_allv(int nbuf, const uint32_t* const* send, uint32_t* const* recv,
                          const int64_t* scnt, const int64_t* soff, const int64_t* rcnt,
                          const int64_t* roff, cudaStream_t s) override {
        g->bufs[rank] = send;
        g->scnt[rank] = scnt;
        g->soff[rank] = soff;
        MG_CU(cudaEventRecord(g->ready[rank], s));
        MG_TRY(lb_barrier(g));
        dc_status st = DC_OK;
        for (int q = 0; q < world; ++q) {
            MG_CU(cudaStreamWaitEvent(s, g->ready[q], 0));
            if (g->scnt[q][rank] != rcnt[q]) {    // finish the protocol, then report
                st = fail(DC_ERR_NCCL, "all-to-all size mismatch between ranks");
                continue;
            }
            for (int b = 0; b < nbuf && rcnt[q] > 0; ++b)
                MG_CU(cudaMemcpyAsync(recv[b] + roff[q], g->bufs[q][b] + g->soff[q][rank],
                                      (size_t)rcnt[q] * 4, cudaMemcpyDeviceToDevice, s));
        }
        MG_TRY(finish(s));
        return st;
    }
};

size_t al256(size_t x) { return (x + 255) / 256 * 256; }

}  // namespace

// ------------------------------------------------------------ runtime state

struct MgCtx {
    Coll* coll = nullptr;
    int rank = 0, world = 1;
    int64_t m = 0;
    // device workspace (splitters, tuples) and the all-to-all receive buffer
    char* ws = nullptr;
    size_t ws_bytes = 0;
    int64_t ws_stride = 0;
    uint32_t *samples = nullptr, *cand = nullptr, *sendbuf = nullptr, *gathered = nullptr;
    int64_t *counts = nullptr, *granks = nullptr, *cmat = nullptr;
    dc_maxsub_tuple *tup = nullptr, *tupall = nullptr;
    dc_maxsub_result* res = nullptr;
    uint32_t* recv = nullptr;
    size_t recv_bytes = 0;
    int64_t* h_pin = nullptr;   // pinned: split matrix, then the max-subarray result
    size_t h_pin_words = 0;
    std::vector<int64_t> last_cmat;
    // fused exchange: the sorted shard lives in xbuf (keys, then values),
    // mapped by every peer; peers[q] = rank q's xbuf in this address space
    int p2p = 0;                // 0 undecided, 1 fused, -1 NCCL all-to-all
    char* xbuf = nullptr;
    std::vector<void*> peers;
    // phase timing (while the plan's kernel timing is on): events around
    // [local sort | splitters | exchange + merge], accumulated per phase
    cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
    double phase_ms[3] = {0, 0, 0};
    int64_t phase_n = 0;
    int64_t moved = 0, moved_total = 0;   // keys this rank received from peers (last / sum)
    ~MgCtx() {
        for (auto e : ev)
            if (e) cudaEventDestroy(e);
        if (coll) coll->unshare(peers);
        if (xbuf) cudaFree(xbuf);
        delete coll;
        if (ws) cudaFree(ws);
        if (recv) cudaFree(recv);
        if (h_pin) cudaFreeHost(h_pin);
    }
};

void mg_destroy(MgCtx* c) { delete c; }
void mg_abort(MgCtx* c) { c->coll->abort(); }

namespace {

dc_status ensure_ws(dc_plan_t p, MgCtx* c, int64_t stride) {
    if (c->ws && c->ws_stride == stride) return DC_OK;
    const int G = c->world;
    const int64_t q = (c->m + stride - 1) / stride;
    const int64_t words = dc_mg_sendbuf_words(G, stride);
    const size_t sz[] = {al256(q * 4),         al256(G * q * 4),          al256(G * q * 8),
                         al256(G * q * 8),     al256(words * 4 + 4),      al256(G * words * 4 + 4),
                         al256(G * (G + 1) * 8), al256(sizeof(dc_maxsub_tuple)),
                         al256(G * sizeof(dc_maxsub_tuple)), al256(sizeof(dc_maxsub_result))};
    size_t total = 0;
    for (size_t v : sz) total += v;
    if (c->ws) cudaFree(c->ws);
    c->ws = nullptr;
    if (cudaMalloc(&c->ws, total) != cudaSuccess) {
        cudaGetLastError();
        return fail(DC_ERR_OUT_OF_MEMORY, "multi-GPU workspace cudaMalloc failed");
    }
    char* at = c->ws;
    auto take = [&](size_t i) {
        char* r = at;
        at += sz[i];
        return r;
    };
    c->samples = (uint32_t*)take(0);
    c->cand = (uint32_t*)take(1);
    c->counts = (int64_t*)take(2);
    c->granks = (int64_t*)take(3);
    c->sendbuf = (uint32_t*)take(4);
    c->gathered = (uint32_t*)take(5);
    c->cmat = (int64_t*)take(6);
    c->tup = (dc_maxsub_tuple*)take(7);
    c->tupall = (dc_maxsub_tuple*)take(8);
    c->res = (dc_maxsub_result*)take(9);
    c->ws_bytes = total;
    c->ws_stride = stride;
    const size_t hw = (size_t)G * (G + 1) + 8;
    if (c->h_pin_words < hw) {
        if (c->h_pin) cudaFreeHost(c->h_pin);
        c->h_pin = nullptr;
        if (cudaMallocHost(&c->h_pin, hw * 8) != cudaSuccess) {
            cudaGetLastError();
            return fail(DC_ERR_OUT_OF_MEMORY, "pinned split-matrix buffer failed");
        }
        c->h_pin_words = hw;
    }
    (void)p;
    return DC_OK;
}

dc_status ensure_recv(MgCtx* c, bool vals) {
    const size_t need = al256((size_t)c->m * 4) * (vals ? 2 : 1);
    if (c->recv_bytes >= need) return DC_OK;
    if (c->recv) cudaFree(c->recv);
    c->recv = nullptr;
    c->recv_bytes = 0;
    if (cudaMalloc(&c->recv, need) != cudaSuccess) {
        cudaGetLastError();
        return fail(DC_ERR_OUT_OF_MEMORY, "all-to-all receive buffer cudaMalloc failed");
    }
    c->recv_bytes = need;
    return DC_OK;
}

// The fused exchange needs every rank to map every peer's shard buffer;
// decided once, collectively (all ranks agree or all use the all-to-all).
dc_status setup_p2p(dc_plan_t p, MgCtx* c) {
    if (c->p2p) return DC_OK;
    int want = p->mg_p2p ? 1 : 0;
    if (const char* e = std::getenv("DC_MG_P2P")) want = std::atoi(e) != 0;
    if (!want) {
        c->p2p = -1;
        return DC_OK;
    }
    const size_t kb = al256((size_t)c->m * 4);
    int ok = 1;
    if (cudaMalloc(&c->xbuf, 2 * kb) != cudaSuccess) {
        cudaGetLastError();
        c->xbuf = nullptr;
        ok = 0;
    }
    int mapped = 0;   // every rank joins the (collective) exchange, even without a buffer
    MG_TRY(c->coll->share_buffer(c->xbuf, c->peers, &mapped, p->stream));
    ok = ok && mapped;
    // agree: the number of ranks that cannot map everything, summed
    MG_TRY(ensure_ws(p, c, c->ws_stride ? c->ws_stride : p->mg_stride));
    c->h_pin[0] = ok ? 0 : 1;
    MG_CU(cudaMemcpyAsync(c->counts, c->h_pin, 8, cudaMemcpyHostToDevice, p->stream));
    MG_TRY(c->coll->all_reduce_sum_i64(c->counts, 1, p->stream));
    MG_CU(cudaMemcpyAsync(c->h_pin, c->counts, 8, cudaMemcpyDeviceToHost, p->stream));
    MG_CU(cudaStreamSynchronize(p->stream));
    if (c->h_pin[0] == 0) {
        c->p2p = 1;
        return DC_OK;
    }
    c->coll->unshare(c->peers);
    if (c->xbuf) cudaFree(c->xbuf);
    c->xbuf = nullptr;
    c->p2p = -1;
    return DC_OK;
}

dc_status mark(dc_plan_t p, MgCtx* c, int i) {
    if (!p->timing) return DC_OK;
    if (!c->ev[i]) MG_CU(cudaEventCreate(&c->ev[i]));
    MG_CU(cudaEventRecord(c->ev[i], p->stream));
    return DC_OK;
}

// keys/vals: this rank's sorted shard (in xbuf when fused); out: the caller's buffers.
dc_status sort_exchange(dc_plan_t p, MgCtx* c, dc_key_type kt, uint32_t* keys, uint32_t* vals,
                        uint32_t* out_k, uint32_t* out_v) {
    const int G = c->world, me = c->rank;
    const int64_t m = c->m, S = p->mg_stride, q = (m + S - 1) / S, wcap = S;
    if ((int64_t)G * wcap * 4 > 200 * 1024)
        return fail(DC_ERR_INVALID_ARG, "world * sample stride * 4 must be <= 200 KiB");
    if ((int64_t)G * q >= (1LL << 24))
        return fail(DC_ERR_INVALID_ARG, "too many splitter candidates; raise the sample stride");
    MG_TRY(ensure_ws(p, c, S));
    const int64_t words = dc_mg_sendbuf_words(G, wcap);
    cudaStream_t s = p->stream;
    // a7: exact composite-order splitters
    MG_TRY(dc_mg_sample(p, keys, m, S, c->samples));
    MG_TRY(c->coll->all_gather(c->samples, c->cand, (size_t)q * 4, s));
    MG_TRY(dc_mg_count(p, kt, keys, m, me, c->cand, q, S, G * q, c->counts));
    MG_CU(cudaMemcpyAsync(c->granks, c->counts, (size_t)G * q * 8, cudaMemcpyDeviceToDevice, s));
    MG_TRY(c->coll->all_reduce_sum_i64(c->granks, (size_t)G * q, s));
    MG_CU(cudaMemsetAsync(c->sendbuf, 0, (size_t)words * 4, s));
    MG_TRY(dc_mg_windows(p, keys, m, me, G, c->counts, c->granks, q, G * q, wcap, c->sendbuf));
    MG_TRY(c->coll->all_gather(c->sendbuf, c->gathered, (size_t)words * 4, s));
    MG_TRY(dc_mg_split_matrix(p, kt, c->gathered, G, m, wcap, c->cmat));
    // the one host sync: split sizes are host arguments of the exchange
    MG_CU(cudaMemcpyAsync(c->h_pin, c->cmat, (size_t)G * (G + 1) * 8, cudaMemcpyDeviceToHost, s));
    int32_t overflow = 0;
    MG_TRY(dc_mg_error(p, &overflow));     // synchronises the plan stream
    if (overflow) return fail(DC_ERR_BAD_STATE, "splitter window overflow (shard not sorted?)");
    const int64_t* cm = c->h_pin;
    c->last_cmat.assign(cm, cm + (size_t)G * (G + 1));
    std::vector<int64_t> scnt(G), soff(G), rcnt(G), roff(G);
    if (dc_mg_exchange_sizes(cm, G, me, m, scnt.data(), soff.data(), rcnt.data(), roff.data()) !=
        DC_OK)
        return fail(DC_ERR_BAD_STATE, std::string("inconsistent split matrix: ") + dc_last_error());
    c->moved = m - rcnt[me];
    c->moved_total += c->moved;
    MG_TRY(mark(p, c, 2));                 // splitters done (host-synchronised above)
    const size_t kb = al256((size_t)m * 4);
    if (c->p2p == 1) {
        // a8+a9 fused: merge straight from the peers' shards (NVLink reads)
        if (G > 4) MG_TRY(ensure_recv(c, vals != nullptr));   // intermediate round
        std::vector<const uint32_t*> rk(G), rv(G);
        std::vector<int64_t> bound(G, m), off(G);
        for (int d = 0; d < G; ++d) {
            rk[d] = (const uint32_t*)c->peers[d];
            rv[d] = (const uint32_t*)((const char*)c->peers[d] + kb);
            off[d] = cm[d * (G + 1) + me];
        }
        uint32_t* tk = G > 4 ? c->recv : nullptr;
        uint32_t* tv = (G > 4 && vals) ? (uint32_t*)((char*)c->recv + kb) : nullptr;
        MG_TRY(dc_mg_merge_peers(p, kt, rk.data(), vals ? rv.data() : nullptr, bound.data(),
                                 off.data(), rcnt.data(), G, tk, tv, out_k, out_v));
        // nobody rewrites its shard (next sort) while a peer may still read it
        return c->coll->barrier(s);
    }
    // a8: all-to-all of the ranges (keys and values in one group)
    MG_TRY(ensure_recv(c, vals != nullptr));
    uint32_t* rk = c->recv;
    uint32_t* rv = vals ? (uint32_t*)((char*)c->recv + kb) : nullptr;
    const uint32_t* send[2] = {keys, vals};
    uint32_t* recv[2] = {rk, rv};
    MG_TRY(c->coll->all_to_allv(vals ? 2 : 1, send, recv, scnt.data(), soff.data(), rcnt.data(),
                                roff.data(), s));
    // a9: local stable G-way merge (earlier ranks win ties) into the caller's buffers
    return dc_mg_merge_runs(p, kt, rk, rv, out_k, out_v, rcnt.data(), G);
}

dc_status attach(dc_plan_t p, Coll* coll, int rank, int world) {
    MgCtx* c = new (std::nothrow) MgCtx();
    if (!c) {
        delete coll;
        return fail(DC_ERR_OUT_OF_MEMORY, "context allocation failed");
    }
    coll->rank = rank;
    coll->world = world;
    c->coll = coll;
    c->rank = rank;
    c->world = world;
    c->m = p->n_global / world;
    p->mg = c;
    p->n = c->m;
    return DC_OK;
}

dc_status can_attach(dc_plan_t p, int32_t rank, int32_t world) {
    if (!p) return fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (p->bad) return fail(DC_ERR_BAD_STATE, "plan poisoned by an earlier CUDA error");
    if (p->mg) return fail(DC_ERR_INVALID_ARG, "plan already has a communicator");
    if (world < 1 || rank < 0 || rank >= world) return fail(DC_ERR_INVALID_ARG, "bad rank/world");
    if (p->n_global % world) return fail(DC_ERR_INVALID_ARG, "n must be divisible by world");
    if (p->scratch || !p->graphs.empty() || p->ms_tiles || p->d_stage || p->mg_state)
        return fail(DC_ERR_INVALID_ARG, "set the communicator before the plan's first run");
    if (p->a != 2 || p->b != 2) return fail(DC_ERR_UNSUPPORTED, "runs need a == b == 2");
    return DC_OK;
}

}  // namespace

dc_status mg_sort(dc_plan_t p, dc_key_type kt, uint32_t* keys, uint32_t* vals) {
    MgCtx* c = p->mg;
    auto run = [&]() -> dc_status {
        if (c->world == 1) return local_sort(p, kt, keys, vals);
        MG_TRY(setup_p2p(p, c));
        MG_TRY(mark(p, c, 0));
        if (c->p2p == 1) {   // levels >= log2 G into the shared shard buffer
            const size_t kb = al256((size_t)c->m * 4);
            uint32_t* xk = (uint32_t*)c->xbuf;
            uint32_t* xv = vals ? (uint32_t*)(c->xbuf + kb) : nullptr;
            MG_TRY(local_sort(p, kt, keys, vals, xk, xv));
            MG_TRY(mark(p, c, 1));
            MG_TRY(sort_exchange(p, c, kt, xk, xv, keys, vals));
        } else {
            MG_TRY(local_sort(p, kt, keys, vals));    // levels >= log2 G: no communication
            MG_TRY(mark(p, c, 1));
            MG_TRY(sort_exchange(p, c, kt, keys, vals, keys, vals));
        }
        MG_TRY(mark(p, c, 3));
        if (p->timing) {                               // accumulate (waits for this sort)
            MG_CU(cudaEventSynchronize(c->ev[3]));
            for (int i = 0; i < 3; ++i) {
                float ms = 0.f;
                MG_CU(cudaEventElapsedTime(&ms, c->ev[i], c->ev[i + 1]));
                c->phase_ms[i] += ms;
            }
            c->phase_n += 1;
        }
        return DC_OK;
    };
    const dc_status st = run();
    if (st != DC_OK) c->coll->abort();
    return st;
}

dc_status mg_maxsub(dc_plan_t p, const int32_t* x, dc_maxsub_result* h_out) {
    MgCtx* c = p->mg;
    auto run = [&]() -> dc_status {
        MG_TRY(ensure_ws(p, c, c->ws_stride ? c->ws_stride : p->mg_stride));
        MG_TRY(dc_run_maxsubarray_tuple_async(p, x, (int64_t)c->rank * c->m, c->tup));
        MG_TRY(c->coll->all_gather(c->tup, c->tupall, sizeof(dc_maxsub_tuple), p->stream));
        MG_TRY(dc_maxsub_combine_async(p, c->tupall, c->world, c->res));
        MG_CU(cudaMemcpyAsync(c->h_pin, c->res, sizeof(dc_maxsub_result), cudaMemcpyDeviceToHost,
                              p->stream));
        MG_CU(cudaStreamSynchronize(p->stream));
        std::memcpy(h_out, c->h_pin, sizeof(dc_maxsub_result));
        return DC_OK;
    };
    const dc_status st = run();
    if (st != DC_OK) c->coll->abort();
    return st;
}

}  // namespace dcx

// ------------------------------------------------------------------- C ABI

extern "C" {

dc_status dc_get_unique_id(uint8_t id[128]) {
    if (!id) return dcx::fail(DC_ERR_INVALID_ARG, "id is NULL");
    const dcx::NcclApi& n = dcx::nccl();
    if (!n.error.empty()) return dcx::fail(DC_ERR_NCCL, n.error);
    ncclUniqueId uid;
    dc_status st = dcx::nccl_check(n.GetUniqueId(&uid), "ncclGetUniqueId");
    if (st != DC_OK) return st;
    std::memcpy(id, &uid, 128);
    return DC_OK;
}

dc_status dc_plan_set_comm(dc_plan_t p, const uint8_t id[128], int32_t rank, int32_t world) {
    dc_status st = dcx::can_attach(p, rank, world);
    if (st != DC_OK) return st;
    if (!id) return dcx::fail(DC_ERR_INVALID_ARG, "id is NULL");
    const dcx::NcclApi& n = dcx::nccl();
    if (!n.error.empty()) return dcx::fail(DC_ERR_NCCL, n.error);
    ncclUniqueId uid;
    std::memcpy(&uid, id, 128);
    auto* coll = new (std::nothrow) dcx::NcclColl();
    if (!coll) return dcx::fail(DC_ERR_OUT_OF_MEMORY, "communicator allocation failed");
    st = dcx::nccl_check(n.CommInitRank(&coll->comm, world, uid, rank), "ncclCommInitRank");
    if (st != DC_OK) {
        coll->comm = nullptr;
        delete coll;
        return st;
    }
    return dcx::attach(p, coll, rank, world);
}

dc_status dc_loopback_create(int32_t world, dc_loopback_t* out) {
    if (!out || world < 1 || world > 1024) return dcx::fail(DC_ERR_INVALID_ARG, "bad arguments");
    *out = nullptr;
    auto* g = new (std::nothrow) dc_loopback_s();
    if (!g) return dcx::fail(DC_ERR_OUT_OF_MEMORY, "group allocation failed");
    g->world = world;
    g->joined.assign(world, false);
    g->ptr.assign(world, nullptr);
    g->bufs.assign(world, nullptr);
    g->scnt.assign(world, nullptr);
    g->soff.assign(world, nullptr);
    g->ready.assign(world, nullptr);
    g->done.assign(world, nullptr);
    for (int r = 0; r < world; ++r) {
        if (cudaEventCreateWithFlags(&g->ready[r], cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&g->done[r], cudaEventDisableTiming) != cudaSuccess) {
            cudaGetLastError();
            dc_loopback_free(g);
            return dcx::fail(DC_ERR_CUDA, "cudaEventCreate failed");
        }
    }
    *out = g;
    return DC_OK;
}

dc_status dc_loopback_free(dc_loopback_t g) {
    if (!g) return DC_OK;
    for (auto e : g->ready)
        if (e) cudaEventDestroy(e);
    for (auto e : g->done)
        if (e) cudaEventDestroy(e);
    delete g;
    return DC_OK;
}

dc_status dc_plan_set_loopback(dc_plan_t p, dc_loopback_t g, int32_t rank) {
    if (!g) return dcx::fail(DC_ERR_INVALID_ARG, "group is NULL");
    dc_status st = dcx::can_attach(p, rank, g->world);
    if (st != DC_OK) return st;
    {
        std::lock_guard<std::mutex> lk(g->mu);
        if (g->joined[rank]) return dcx::fail(DC_ERR_INVALID_ARG, "rank already joined");
        g->joined[rank] = true;
    }
    auto* coll = new (std::nothrow) dcx::LoopColl();
    if (!coll) return dcx::fail(DC_ERR_OUT_OF_MEMORY, "communicator allocation failed");
    coll->g = g;
    return dcx::attach(p, coll, rank, g->world);
}

dc_status dc_plan_comm_info(dc_plan_t p, int32_t* rank, int32_t* world, int64_t* shard_n) {
    if (!p) return dcx::fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (rank) *rank = p->mg ? p->mg->rank : 0;
    if (world) *world = p->mg ? p->mg->world : 1;
    if (shard_n) *shard_n = p->n;
    return DC_OK;
}

dc_status dc_plan_set_mg_stride(dc_plan_t p, int64_t stride) {
    if (!p) return dcx::fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (stride < 1 || stride > (1 << 20)) return dcx::fail(DC_ERR_INVALID_ARG, "stride out of range");
    p->mg_stride = stride;
    return DC_OK;
}

dc_status dc_plan_set_mg_p2p(dc_plan_t p, int32_t enable) {
    if (!p) return dcx::fail(DC_ERR_INVALID_ARG, "plan is NULL");
    if (p->mg && p->mg->p2p != 0)
        return dcx::fail(DC_ERR_INVALID_ARG, "exchange mode is fixed after the first sort");
    p->mg_p2p = enable != 0;
    return DC_OK;
}

dc_status dc_plan_mg_exchange_mode(dc_plan_t p, int32_t* mode) {
    if (!p || !mode) return dcx::fail(DC_ERR_INVALID_ARG, "NULL argument");
    *mode = p->mg ? p->mg->p2p : 0;
    return DC_OK;
}

dc_status dc_plan_mg_phase_times(dc_plan_t p, double* h_ms3, int64_t* sorts,
                                 int64_t* keys_received) {
    if (!p || !h_ms3) return dcx::fail(DC_ERR_INVALID_ARG, "NULL argument");
    if (!p->mg) return dcx::fail(DC_ERR_INVALID_ARG, "plan has no communicator");
    for (int i = 0; i < 3; ++i) h_ms3[i] = p->mg->phase_ms[i];
    if (sorts) *sorts = p->mg->phase_n;
    if (keys_received) *keys_received = p->mg->moved_total;
    return DC_OK;
}

dc_status dc_plan_mg_reset_phases(dc_plan_t p) {
    if (!p || !p->mg) return dcx::fail(DC_ERR_INVALID_ARG, "plan has no communicator");
    for (double& v : p->mg->phase_ms) v = 0;
    p->mg->phase_n = 0;
    p->mg->moved_total = 0;
    return DC_OK;
}

dc_status dc_mg_exchange_sizes(const int64_t* cm, int32_t world, int32_t rank, int64_t shard_n,
                               int64_t* scnt, int64_t* soff, int64_t* rcnt, int64_t* roff) {
    if (!cm || !scnt || !soff || !rcnt || !roff || world < 1 || rank < 0 || rank >= world ||
        shard_n < 0)
        return dcx::fail(DC_ERR_INVALID_ARG, "bad exchange-size arguments");
    const int G = world;
    for (int r = 0; r < G; ++r) {
        if (cm[r * (G + 1)] != 0 || cm[r * (G + 1) + G] != shard_n)
            return dcx::fail(DC_ERR_INVALID_ARG, "split-matrix row must run from 0 to shard_n");
        for (int d = 0; d < G; ++d)
            if (cm[r * (G + 1) + d + 1] < cm[r * (G + 1) + d])
                return dcx::fail(DC_ERR_INVALID_ARG, "split-matrix row not monotone");
    }
    int64_t tot = 0;
    for (int d = 0; d < G; ++d) {
        soff[d] = cm[rank * (G + 1) + d];                       // my elements for rank d
        scnt[d] = cm[rank * (G + 1) + d + 1] - soff[d];
        rcnt[d] = cm[d * (G + 1) + rank + 1] - cm[d * (G + 1) + rank];   // rank d's for me
        roff[d] = tot;                                          // runs land in rank order
        tot += rcnt[d];
    }
    if (tot != shard_n)
        return dcx::fail(DC_ERR_INVALID_ARG, "received element count != shard size");
    return DC_OK;
}

dc_status dc_plan_last_splits(dc_plan_t p, int64_t* h_cmat) {
    if (!p || !h_cmat) return dcx::fail(DC_ERR_INVALID_ARG, "NULL argument");
    if (!p->mg || p->mg->last_cmat.empty())
        return dcx::fail(DC_ERR_INVALID_ARG, "no multi-GPU sort has run on this plan");
    std::memcpy(h_cmat, p->mg->last_cmat.data(), p->mg->last_cmat.size() * 8);
    return DC_OK;
}

}  // extern "C"
