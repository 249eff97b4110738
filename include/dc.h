/*
 * dc.h -- C ABI of the B200-native breadth-first divide-and-conquer library.
 *
 * The operation: the breadth-first, level-by-level execution of a recursive
 * divide-and-conquer T(n) = aT(n/b) + f(n) (Sec. 4, P:L229-306;
 * Alg 2): all a^i subproblems of size n/b^i at level i run in one
 * data-parallel step, base cases first, then one combine pass per level,
 * bottom-up.  Two instances:
 *   - mergesort, a = b = 2, linear stable merge combine (Alg 6 P:L623-630,
 *     Alg 7);
 *   - maximum-subarray-sum with an O(1) combine (north star; the O(1)-combine
 *     pattern of Alg 4/5).
 * "P:Lx-y" = lines of PAPER.md (the paper text).
 *
 * Conventions (all entry points)
 *   - No exception crosses the ABI; every call returns a dc_status.
 *   - Validation failures return before any device work; inputs untouched.
 *   - Device pointers are plain CUDA device pointers on the device that was
 *     current when the plan first ran (the "plan device"); 4-byte elements,
 *     16-byte aligned (misalignment -> DC_ERR_INVALID_ARG).  Host pointers
 *     are ordinary host memory (pinned or pageable).
 *   - Ownership: the caller owns every buffer passed in.  The plan owns its
 *     scratch (allocated lazily on first run unless dc_plan_set_scratch gave
 *     one), its partition arrays and its CUDA graphs; dc_free releases them.
 *   - Asynchrony: dc_run_mergesort and the *_async calls only enqueue work on
 *     the plan stream (default: the legacy default stream) and return.  Calls
 *     that return a result through a host pointer synchronise the stream.
 *     An asynchronous CUDA fault surfaces as DC_ERR_CUDA on a later call; the
 *     plan is then in DC_ERR_BAD_STATE and must be freed.
 *   - A plan is used by one host thread at a time.
 *   - dc_last_error() returns a thread-local human-readable detail string for
 *     the last non-OK status returned on this thread.
 */
#ifndef DC_H
#define DC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    DC_OK = 0,
    DC_ERR_INVALID_ARG = 1,   /* bad size, NULL, misaligned pointer, ...     */
    DC_ERR_UNSUPPORTED = 2,   /* valid request this build cannot run (a!=2) */
    DC_ERR_OUT_OF_MEMORY = 3, /* scratch allocation failed                    */
    DC_ERR_CUDA = 4,          /* a CUDA runtime call or kernel failed        */
    DC_ERR_NCCL = 5,          /* NCCL missing or a collective failed         */
    DC_ERR_BAD_STATE = 6      /* plan poisoned by an earlier CUDA error       */
} dc_status;

typedef enum {
    DC_KEY_U32 = 0, /* uint32 keys                                           */
    DC_KEY_I32 = 1, /* int32 keys                                            */
    DC_KEY_F32 = 2  /* float32 keys compared with '<' only: +0.0 == -0.0 keep
                       input order; NaN is a precondition violation.         */
} dc_key_type;

typedef struct dc_plan_s *dc_plan_t; /* opaque */

/* Result of the max-subarray instance: the non-empty subarray x[start..end]
 * (inclusive, 0-based, global indices) of maximum int64 sum; among several
 * maxima the lexicographically smallest (start, end) (R9-R10). */
typedef struct {
    int64_t sum;
    int64_t start;
    int64_t end;
} dc_maxsub_result;

/* The O(1)-combine summary of a contiguous segment [l, r]:
 * tot = sum; pre = max prefix sum (ends at pe, smallest end on ties);
 * suf = max suffix sum (starts at ss, smallest start); best = max subarray
 * (bs..be, lexicographically smallest).  Indices are global.  Used to combine
 * per-rank results of a sharded max-subarray in rank order. */
typedef struct {
    int64_t tot, pre, suf, best;
    int64_t pe, ss, bs, be;
} dc_maxsub_tuple;

/* ------------------------------------------------------------------ plans */

/* dc_plan: describe the recursion T(n) = aT(n/b) + f(n) for an input
 * of n elements whose recursion stops at subproblems of size <= base_size.
 * Host-only (no device work).  n >= 1, 2 <= a,b <= 1024, 1 <= base_size <= n,
 * n <= 2^31-1.  Runs need a == b == 2 (mergesort and max-subarray);
 * other (a, b) only serve level-table queries (DC_ERR_UNSUPPORTED at run).
 * base_size changes only the level table, never a result. */
dc_status dc_plan(int64_t n, int32_t a, int32_t b, int64_t base_size, dc_plan_t *out);

/* Level table of the plan: level i (0 = root) has nodes[i] = a^i
 * subproblems of size sizes[i] = ceil(n / b^i); the last level L is the first
 * whose size is <= base_size.  Writes *num_levels = L + 1 and, if the arrays
 * are non-NULL, min(L+1, capacity) entries of each. */
dc_status dc_plan_levels(dc_plan_t plan, int32_t *num_levels, int64_t *nodes,
                         int64_t *sizes, int32_t capacity);

/* Execution schedule of an a=b=2 sort of this key type (with or without
 * values) as dc_run_mergesort will run it: the fused bottom kernel sorts tiles
 * of `tile` keys (the leaves plus fused_levels = ceil(log2(tile)) levels of
 * the binary tree, entirely on chip); global_passes =
 * ceil(log2(ceil(n/tile))) levels remain, executed in hbm_passes passes over
 * HBM (one or two levels per pass).  Tile class and pass kind are the
 * planner's choice (dc_model_sort_schedule) unless forced with
 * dc_plan_set_tile_class / dc_plan_set_two_level; with NK1 cluster levels
 * (dc_plan_set_nk1_cluster) `tile` is the cluster's fused run width.  Any
 * output pointer may be NULL. */
dc_status dc_plan_schedule(dc_plan_t plan, dc_key_type key_type, int32_t with_vals,
                           int32_t *tile, int32_t *fused_levels, int32_t *global_passes,
                           int32_t *hbm_passes);

/* Force (1) or forbid (0) the two-levels-per-pass schedule (every
 * pass merges groups of four runs -- an exact 4-run selection per output
 * tile, then a 4-way tile merge; sort4_kernels.cuh), or leave it to the
 * planner (-1, default).  Results are identical either way. */
dc_status dc_plan_set_two_level(dc_plan_t plan, int32_t enable);

/* Force the NK1 tile class (1 quarter-size tiles of 128-thread CTAs, 2 full
 * tiles) or leave it to the planner (0, default).  Results are identical. */
dc_status dc_plan_set_tile_class(dc_plan_t plan, int32_t tile_class);

/* NK1 cluster levels for keys-only u32/i32 sorts: a cluster of cs
 * CTAs (cs = 2, 4, 8 or 16; a thread-block cluster, distributed shared
 * memory) sorts cs adjacent tiles and runs log2(cs) more merge levels of Alg 7
 * on chip -- every CTA gathers the inputs of its output range
 * from its partners' shared memory, then merges locally -- so the fused runs
 * are cs tiles wide and log2(cs) global levels fewer remain.  cs = 1 turns it
 * off, 0 (default) leaves it to the planner's rule (small sorts, where every
 * global level is a latency-bound launch).  Key-value and
 * f32 sorts ignore it.  Results are identical.  DC_ERR_INVALID_ARG for any
 * other cs. */
dc_status dc_plan_set_nk1_cluster(dc_plan_t plan, int32_t cs);

/* Enable (default) or disable the fused partition of L2-resident sorts (n <
 * 2^23): every one-level merge CTA finds the co-ranks of its own output tile
 * (two 33-ary warp searches, Alg 3's fn(id, param) inside the merge kernel,
 * P:L325-332) instead of a separate NK2 launch per level.  Results are
 * identical either way. */
dc_status dc_plan_set_fused_partition(dc_plan_t plan, int32_t enable);

/* Enable (default) or disable CUDA-graph replay of the sort's launch sequence:
 * the first dc_run_mergesort for a given (keys, vals, key type) runs eagerly,
 * the second captures a graph, later ones replay it.  Disabled automatically
 * while per-kernel timing is on.  Results are identical. */
dc_status dc_plan_set_graphs(dc_plan_t plan, int32_t enable);

/* Chunked pipeline of the one-level schedule (default 1 = off; measured slower
 * on B200):
 * the array is cut into chunks of tile*2^k keys; each chunk's fused bottom
 * levels and in-chunk merge levels run on a stream of their own, so chunks
 * overlap (one chunk's HBM-bound merges with the next one's compute-bound
 * NK1); the top log2(chunks) levels follow on the plan stream.  Not used
 * while per-kernel timing is on.  Results are identical. */
dc_status dc_plan_set_pipeline(dc_plan_t plan, int32_t chunks);

/* Stream all device work of this plan is enqueued on (a cudaStream_t). */
dc_status dc_plan_set_stream(dc_plan_t plan, void *cuda_stream);

/* Scratch the sort needs: n*4 bytes for keys (+ n*4 for values) ping-pong
 * (the paper's 2n working space) plus the partition array. */
dc_status dc_plan_scratch_bytes(dc_plan_t plan, int32_t with_vals, size_t *bytes);

/* Optional caller-owned scratch (device, 16-byte aligned, >= the size above).
 * Without it the plan allocates its own on first use. */
dc_status dc_plan_set_scratch(dc_plan_t plan, void *d_scratch, size_t bytes);

/* Frees the plan and everything it owns.  Accepts NULL. */
dc_status dc_free(dc_plan_t plan);

/* ------------------------------------------------------------- mergesort */

/* In-place stable sort of d_keys[0..n) (device), permuting d_vals[0..n)
 * (device, nullable) with the keys.  Alg 7 executed bottom-up: fused bottom
 * levels, then one merge-path pass per remaining level.  Enqueues only. */
dc_status dc_run_mergesort(dc_plan_t plan, dc_key_type key_type, void *d_keys,
                           uint32_t *d_vals);

/* Same, host buffers: copies h_keys (+h_vals) to device memory owned by the
 * plan, sorts, copies back, synchronises.  End-to-end entry point. */
dc_status dc_run_mergesort_host(dc_plan_t plan, dc_key_type key_type, void *h_keys,
                                uint32_t *h_vals);

/* Streaming end-to-end sorts of HOST buffers (pinned for overlap).  Each
 * submission copies h_in_keys (+h_in_vals) into one of three plan-owned device
 * slots, sorts there and copies the result to h_out_keys (+h_out_vals); the
 * host input is not modified.  Work of consecutive submissions overlaps: the
 * upload of one, the sort of the previous and the download of the one before
 * run on separate streams (PCIe is full duplex).  A submission starts after
 * the work already enqueued on the plan stream, and every later run of the
 * plan that uses its scratch (dc_run_mergesort, dc_mg_merge_*) is ordered on
 * the plan stream after the submitted sorts.  Returns after enqueueing;
 * the host buffers must stay valid until dc_sort_host_wait returns. */
dc_status dc_sort_host_submit(dc_plan_t plan, dc_key_type key_type, const void *h_in_keys,
                              const uint32_t *h_in_vals, void *h_out_keys, uint32_t *h_out_vals);

/* Waits (host) until every submitted host sort has written its output; the
 * plan stream is also made to wait for them. */
dc_status dc_sort_host_wait(dc_plan_t plan);

/* ----------------------------------------------------------- max-subarray */

/* Max subarray of d_x[0..n) (device int32).  Synchronises; writes *h_out. */
dc_status dc_run_maxsubarray(dc_plan_t plan, const int32_t *d_x, dc_maxsub_result *h_out);

/* Enqueue-only variant: writes the result (dc_maxsub_result, device memory)
 * to d_out; index_offset is added to every index (a shard's global start). */
dc_status dc_run_maxsubarray_async(dc_plan_t plan, const int32_t *d_x, int64_t index_offset,
                                   dc_maxsub_result *d_out);

/* Enqueue-only: the segment summary tuple of d_x[0..n) with indices offset by
 * index_offset, written to d_tuple (device). */
dc_status dc_run_maxsubarray_tuple_async(dc_plan_t plan, const int32_t *d_x,
                                         int64_t index_offset, dc_maxsub_tuple *d_tuple);

/* Enqueue-only: ordered combine of count tuples (device; tuple r covers the
 * segment left of tuple r+1) into one result (device). */
dc_status dc_maxsub_combine_async(dc_plan_t plan, const dc_maxsub_tuple *d_tuples,
                                  int32_t count, dc_maxsub_result *d_out);

/* Host buffers end to end: copy h_x to the device, run, return the result. */
dc_status dc_run_maxsubarray_host(dc_plan_t plan, const int32_t *h_x, dc_maxsub_result *h_out);

/* ---------------------------------------------- D&C sum */
/* The paper's own D&C example, Alg 4: sum(a, size) recurses on
 * the halves and combines with a[0] += a[size/2].  Third instance of the
 * breadth-first O(1)-combine template include/dc_reduce.cuh (also usable
 * with user monoids from CUDA code). */

/* Exact int64 sum of d_x[0..n) (device int32).  Synchronises; *h_out. */
dc_status dc_run_sum(dc_plan_t plan, const int32_t *d_x, int64_t *h_out);

/* Enqueue-only variant writing the int64 result to device memory d_out. */
dc_status dc_run_sum_async(dc_plan_t plan, const int32_t *d_x, int64_t *d_out);

/* Alg 5 literally: one kernel launch per level, the id-th of m
 * work-items computes a[id] <- a[id] + a[id+m]; d_work (device int64, n
 * elements) is overwritten; synchronises and returns a[0] in *h_out. */
dc_status dc_run_sum_alg5(dc_plan_t plan, int64_t *d_work, int64_t *h_out);

/* ------------------------------------- work-division model */
/* The paper's advanced hybrid work division (Sec. 5.2) for a D&C
 * with f(m) = m^{log_b a} (mergesort: a = b = 2) on an HPU with p CPU cores,
 * g GPU cores and CPU/GPU speed ratio gamma (0 < gamma < 1; Sec. 3.2).  A
 * fraction alpha of the subproblems runs on the CPU; the GPU runs the rest
 * from the leaves up to level y where both finish together (the closed forms
 * of Sec. 5.2.2, three cases).  Host-only; INVALID_ARG for a,b < 2, p < 1,
 * g < 1, gamma outside (0,1), n < 2 or alpha outside [p/n^{log_b a}, 1). */

/* GPU share of the total work n^{log_b a}(log_b n + 1) for a given alpha, the
 * level y reached by the GPU and the case (1, 2, 3) of Tg that applies. */
dc_status dc_model_gpu_work(int32_t a, int32_t b, int32_t p, double g, double gamma, double n,
                            double alpha, double *gpu_work_fraction, double *level_y,
                            int32_t *model_case);

/* alpha* maximising the GPU work ("numeric methods") and the
 * corresponding share, level y and case.  The paper's example (a=b=2, p=4,
 * g=2^12, gamma=1/160, n=2^24) gives alpha* ~ 0.16, ~52 %, y ~ 10. */
dc_status dc_model_optimise(int32_t a, int32_t b, int32_t p, double g, double gamma, double n,
                            double *alpha, double *gpu_work_fraction, double *level_y,
                            int32_t *model_case);

/* B200 schedule planner: the Sec. 5.2 analysis re-parameterised
 * for one B200 (model.cu).  The levels of the recursion tree run on chip (the
 * bottom ceil(log2 T) levels of every NK1 tile, T set by the tile class) or
 * in HBM passes of one level (NK2 + NK3) or two levels (NK2-4 + NK3-4); each
 * kernel costs a launch term plus waves of resident CTAs (the parallelism
 * threshold), with L2- and HBM-resident wave times fitted to
 * B200 measurements (tools/planner_sweep.py, tools/planner_fit.py,
 * profiles/r02/planner_sweep.json).  dc_run_mergesort runs the candidate of
 * least predicted time unless the plan forces a tile class or pass kind.
 * candidates_ms: [quarter tiles, one level/pass], [quarter, two], [full,
 * one], [full, two].  Host-only; INVALID_ARG on bad arguments. */
typedef struct {
    int32_t tile_class;      /* 1 quarter-size tiles, 2 full tiles */
    int32_t two_level;       /* 1: two tree levels per HBM pass (4-way passes) */
    int32_t tile;            /* keys per NK1 tile */
    int32_t fused_levels;    /* ceil(log2 tile) levels on chip */
    int32_t global_levels;   /* ceil(log2(n / tile)) levels above the tile */
    int32_t hbm_passes;      /* HBM passes of the chosen schedule */
    double predicted_ms;
    double candidates_ms[4];
} dc_sort_schedule;
/* tile_class: 0 free, 1 or 2 forced; two_level: -1 free, 0 or 1 forced. */
dc_status dc_model_sort_schedule(int64_t n, dc_key_type key_type, int32_t with_vals,
                                 int32_t tile_class, int32_t two_level, dc_sort_schedule *out);

/* ------------------------------------------------ multi-GPU (rows a7-a10) */
/* One process (or, for tests, one thread) per GPU.  With a communicator set,
 * the plan's n is the GLOBAL problem size; every rank passes its shard of
 * m = n/world elements, the global positions [rank*m, (rank+1)*m):
 *   dc_run_mergesort   sorts the shard locally (levels >= log2 world), then
 *                      runs the top log2(world) levels of the merge tree as
 *                      ONE exchange ("could easily be extended to
 *                      multiple gpu cards"; the single-transfer principle of
 *                      P:L474-478): exact composite-order splitters from an
 *                      all-gather of samples, an all-reduce of their counts and
 *                      an all-gather of bracketing windows; one host sync for
 *                      the split sizes; one all-to-all of keys (+ values); a
 *                      local stable G-way merge.  On exit rank r holds global
 *                      positions [r*m, (r+1)*m) of the stable sorted order.
 *   dc_run_maxsubarray returns the global result (indices are global
 *                      positions): per-rank summary tuple -> all-gather ->
 *                      ordered combine.
 * Collectives are enqueued on the plan stream.  All ranks must make the same
 * calls in the same order.  Host-buffer entry points are single-GPU only
 * (DC_ERR_UNSUPPORTED with a communicator). */

/* 128 opaque bytes identifying a new NCCL communicator; create on one rank and
 * broadcast (e.g. torch.distributed.broadcast_object_list).  NCCL is loaded
 * at run time (the copy already in the process, else libnccl.so.2, else
 * $DC_NCCL_LIB); DC_ERR_NCCL if it cannot be. */
dc_status dc_get_unique_id(uint8_t id[128]);

/* Joins the NCCL communicator `id` as `rank` of `world` (collective: blocks
 * until every rank has joined; call with the plan's device current).  Must
 * precede the plan's first run; n % world == 0 required (DC_ERR_INVALID_ARG).
 * world == 1 is allowed (the single-GPU path). */
dc_status dc_plan_set_comm(dc_plan_t plan, const uint8_t id[128], int32_t rank, int32_t world);

/* In-process loopback group: `world` ranks that are threads of one process
 * sharing one GPU, with the collectives done by device copies between their
 * buffers.  Same protocol and kernels as NCCL; used to test the multi-GPU path
 * on a single GPU.  Free after every member plan has been freed. */
typedef struct dc_loopback_s *dc_loopback_t;
dc_status dc_loopback_create(int32_t world, dc_loopback_t *out);
dc_status dc_loopback_free(dc_loopback_t group);
/* Joins `group` as `rank` (not collective).  Same preconditions as
 * dc_plan_set_comm.  A member that fails aborts the group: the others then
 * return DC_ERR_NCCL instead of waiting (and after 120 s in any case). */
dc_status dc_plan_set_loopback(dc_plan_t plan, dc_loopback_t group, int32_t rank);

/* Communicator of a plan: rank, world and shard size m (1, 0, n without). */
dc_status dc_plan_comm_info(dc_plan_t plan, int32_t *rank, int32_t *world, int64_t *shard_n);

/* Sample stride S of the splitter search (default 4096; windows hold < S keys;
 * world*S*4 <= 200 KiB).  Set before a run, the same on every rank. */
dc_status dc_plan_set_mg_stride(dc_plan_t plan, int64_t stride);

/* Exchange of the multi-GPU sort.  enable != 0: FUSED -- every rank sorts
 * its shard into a plan-owned buffer that all peers map (CUDA IPC over
 * NVLink/NVSwitch; plain pointers in a loopback group), and the first round
 * of the G-way merge reads the runs straight from the peers' buffers
 * (dc_mg_merge_peers: up to four peers per 4-way pass), then a stream-ordered
 * barrier; no all-to-all, no receive buffer write.  enable == 0 (default
 * until the fused mode has been measured across GPUs): NCCL all-to-all
 * (grouped send/recv), then the local merge (dc_mg_merge_runs).
 * Set before the first sort, the same on every rank; if any rank cannot map
 * every peer, all ranks fall back to the all-to-all (decided collectively at
 * the first sort).  $DC_MG_P2P=0/1 overrides. */
dc_status dc_plan_set_mg_p2p(dc_plan_t plan, int32_t enable);

/* Exchange in use: 1 fused, -1 all-to-all, 0 not decided yet / no communicator. */
dc_status dc_plan_mg_exchange_mode(dc_plan_t plan, int32_t *mode);

/* Phase times of the multi-GPU sorts run while dc_plan_enable_timing is on
 * (CUDA events on the plan stream; each timed sort waits for itself):
 * h_ms3[0] local sort (levels >= log2 G), [1] splitters incl. the host sync,
 * [2] exchange + G-way merge (fused, or all-to-all + merge), summed over
 * *sorts sorts; *keys_received = keys this rank took from peers (summed). */
dc_status dc_plan_mg_phase_times(dc_plan_t plan, double *h_ms3, int64_t *sorts,
                                 int64_t *keys_received);
dc_status dc_plan_mg_reset_phases(dc_plan_t plan);

/* Split matrix of the last multi-GPU sort: h_cmat[r*(world+1) + d] = number of
 * rank-r elements among the first d*m of the global stable order. */
dc_status dc_plan_last_splits(dc_plan_t plan, int64_t *h_cmat);

/* ------------------------------------------- multi-GPU building blocks */
/* The top log2(G) levels of a G-way sharded sort (not in
 * the paper, which notes the method "could easily be extended to multiple gpu
 * cards").  Rank r holds global positions [r*m, (r+1)*m) and has
 * sorted them with dc_run_mergesort.  These are the per-rank device steps
 * of the protocol above, exposed for callers that run the collectives
 * themselves (e.g. in torch.distributed; dist.py).  All are enqueue-only on the plan stream unless stated.
 * Composite order: element (key, rank, position) -- the global stable order.
 */

/* Words of one rank's splitter send buffer for `world` ranks and windows of
 * wcap keys: 6*(world-1) header words (three int64 per boundary) followed by
 * (world-1)*wcap key words, rounded up to a multiple of 4 words so that
 * back-to-back buffers of all ranks stay 16-byte aligned for any wcap.
 * 0 if world < 2. */
int64_t dc_mg_sendbuf_words(int32_t world, int64_t wcap);

/* Samples of a sorted shard: d_samples[j] = d_keys[j*stride] for
 * j < ceil(n/stride). */
dc_status dc_mg_sample(dc_plan_t plan, const uint32_t *d_keys, int64_t n, int64_t stride,
                       uint32_t *d_samples);

/* Composite counts.  d_cand holds the all-gathered samples of every rank,
 * rank-major (candidate c = owner*per_rank + j is the element at position
 * j*stride of rank `owner`), cands = world*per_rank < 2^24.  Writes, for
 * every candidate, the number of elements of this rank's sorted shard
 * d_keys[0..n) strictly below it in composite order (int64 d_counts[c]).
 * Summing d_counts over ranks gives every candidate's global position. */
dc_status dc_mg_count(dc_plan_t plan, dc_key_type key_type, const uint32_t *d_keys, int64_t n,
                      int32_t rank, const uint32_t *d_cand, int64_t per_rank, int64_t stride,
                      int64_t cands, int64_t *d_counts);

/* Splitter windows.  d_ranks: global positions of the candidates (the
 * all-reduced sum of every rank's d_counts).  For every boundary k_d = d*n,
 * d = 1..world-1, brackets k_d between two consecutive candidates and writes
 * into d_sendbuf (dc_mg_sendbuf_words words) this rank's elements strictly
 * between them (< stride of them, window capacity wcap >= stride) with
 * {lo, len, t}: their shard range and how many window elements of all ranks
 * belong to the first k_d. */
dc_status dc_mg_windows(dc_plan_t plan, const uint32_t *d_keys, int64_t n, int32_t rank,
                        int32_t world, const int64_t *d_counts, const int64_t *d_ranks,
                        int64_t per_rank, int64_t cands, int64_t wcap, uint32_t *d_sendbuf);

/* Exact split matrix from the all-gathered send buffers of all ranks (rank
 * order, back to back): d_cmat[r*(world+1) + d] = number of rank-r elements
 * among the first d*shard_n of the global stable order (d = 0..world).
 * Requires world*wcap*4 <= 200 KiB. */
dc_status dc_mg_split_matrix(dc_plan_t plan, dc_key_type key_type, const uint32_t *d_gathered,
                             int32_t world, int64_t shard_n, int64_t wcap, int64_t *d_cmat);

/* Host-only: the exchange plan of `rank` from a split matrix h_cmat
 * (world x (world+1), as dc_mg_split_matrix / dc_plan_last_splits give it).
 * Rank `rank` sends its shard range [send_off[d], send_off[d] + send_cnt[d])
 * to rank d and receives recv_cnt[d] elements from rank d, placed at
 * recv_off[d] of its receive buffer (runs back to back in rank order, the
 * order dc_mg_merge_runs needs for the global stable order).  Checks that
 * every row runs monotonically from 0 to shard_n and that the received total
 * is shard_n (INVALID_ARG otherwise).  Output arrays hold `world` entries.
 * This is the runtime's own host step (dc_run_mergesort with a communicator
 * calls it); exposed so that callers and tests can drive it. */
dc_status dc_mg_exchange_sizes(const int64_t *h_cmat, int32_t world, int32_t rank,
                               int64_t shard_n, int64_t *send_cnt, int64_t *send_off,
                               int64_t *recv_cnt, int64_t *recv_off);

/* Synchronises and reports whether a window overflowed its capacity
 * (*h_err != 0 means the shard was not sorted or wcap < stride). */
dc_status dc_mg_error(dc_plan_t plan, int32_t *h_err);

/* Local stable merge of `runs` sorted runs stored back to back in d_in_keys
 * (run r has h_run_len[r] elements, host array; total <= plan n) into
 * d_out_keys; earlier runs win ties (Alg 7's top levels).
 * Values (nullable, both or neither) move with their keys.  Groups of four
 * runs merge in one HBM pass (exact 4-run selection + 4-way tile merge),
 * a pair in one pass: ceil(log4 runs) passes.  d_in_* is used as ping-pong
 * space (with more than 16 runs) and may be clobbered. */
dc_status dc_mg_merge_runs(dc_plan_t plan, dc_key_type key_type, uint32_t *d_in_keys,
                           uint32_t *d_in_vals, uint32_t *d_out_keys, uint32_t *d_out_vals,
                           const int64_t *h_run_len, int32_t runs);

/* a8+a9 fused: stable merge of `runs` sorted runs that live in separate
 * buffers -- in the multi-GPU sort, the sorted shards of the peer GPUs, read
 * directly over NVLink, so the exchange overlaps the merge tile by tile and
 * no receive buffer is written.  Run r is h_len[r] elements at offset
 * h_off[r] of the buffer h_run_keys[r] (+ h_run_vals[r]; host arrays of
 * device pointers, 16-byte aligned, readable for h_bound[r] elements; the
 * pointers may be peer mappings).  Earlier runs win ties.  Output:
 * d_out_keys (+ d_out_vals), sum(h_len) <= plan n elements.  Up to four runs
 * merge in ONE pass straight from their buffers (4-way tiles whose pieces the
 * TMA fetches from up to four peers); with more than four runs the first
 * round writes d_tmp_* (n elements each) and later rounds are local.
 * Enqueue-only. */
dc_status dc_mg_merge_peers(dc_plan_t plan, dc_key_type key_type,
                            const uint32_t *const *h_run_keys, const uint32_t *const *h_run_vals,
                            const int64_t *h_bound, const int64_t *h_off, const int64_t *h_len,
                            int32_t runs, uint32_t *d_tmp_keys, uint32_t *d_tmp_vals,
                            uint32_t *d_out_keys, uint32_t *d_out_vals);

/* ------------------------------------------------------ instrumentation */

/* Kernel classes for dc_plan_kernel_time. */
#define DC_KERNEL_NK1_BLOCKSORT 0 /* fused bottom levels              */
#define DC_KERNEL_NK2_PARTITION 1 /* co-ranks of one pass (2- or 4-run) */
#define DC_KERNEL_NK3_MERGE 2     /* one HBM merge pass (1 or 2 levels) */
#define DC_KERNEL_NK4_MAXSUB 3    /* max-subarray tiles + top combine */
#define DC_KERNEL_COUNT 4

/* Turn per-launch CUDA-event timing on (1) or off (0); resets the totals.
 * When on, every kernel launch is bracketed by two events on the plan stream. */
dc_status dc_plan_enable_timing(dc_plan_t plan, int32_t enable);

/* Total device time (ms) and number of timed launches of one kernel class
 * since timing was enabled.  Waits for the pending events. */
dc_status dc_plan_kernel_time(dc_plan_t plan, int32_t kernel, double *total_ms,
                              int64_t *launches);

/* ------------------------------------------------------------- misc */

const char *dc_status_string(dc_status s);
const char *dc_last_error(void);
/* Number of kernels this plan launched since creation (instrumentation). */
int64_t dc_plan_launch_count(dc_plan_t plan);
/* Library version string. */
const char *dc_version(void);

#ifdef __cplusplus
}
#endif
#endif /* DC_H */
