// ctx.h — device context of one rank and the small device helpers shared by the kernels.
#pragma once
#include <cuda.h>  // CUtensorMap (type only: the encoder is resolved through cudaGetDriverEntryPoint)
#include <cuda_runtime.h>

#include <cstdint>
#include <vector>

#include "moment.h"
#include "status.h"

struct moment_ctx_s {
    int32_t rank = 0, world = 1, device = 0;
    int64_t n_vertices = 0;
    int64_t max_seeds = 0;
    int32_t max_hops = 0;
    std::vector<int32_t> max_fanout;
    std::vector<int64_t> max_F;  // per hop h = 0..max_hops: bound on |F_h|
    std::vector<int64_t> max_E;  // per hop: bound on E_h
    int64_t max_nodes = 0, max_edges = 0, max_offsets = 0;
    int64_t row_bytes = 0, row_stride = 0;
    int32_t n_bins = 0;
    int32_t gather_path = 0;  // 0 auto (TMA bulk copies for local rows), 1 LDG.128 only, 2 bulk, 3 tma4 (MOMENT_GATHER_PATH)
    // tile::gather4 tensor map of the replicated table (built on first use) and its L2 promotion
    CUtensorMap tma_map{};
    const void* tma_base = nullptr;
    // L2 promotion of the gathered rows: 64 B (measured: a 400-byte row then costs 448 B of DRAM reads instead
    // of the 512 B whole 128-byte lines the default fetches; MOMENT_TMA_PROMO: 0 none, 1 64B, 2 128B, 3 256B)
    int32_t tma_promo = 1;
    // gather4 launch shape: 1-warp blocks of 4 stages x tma4_rows rows, tma4_blocks_per_sm per SM (MOMENT_TMA4_BLOCKS,
    // MOMENT_TMA4_ROWS = 8 / 16 / 32). A lone launch streams faster with more issuing warps per SM (1: 0.55 of the
    // copy peak, 2: 0.61-0.73, 3-4: 0.72-0.74), while inside the saturated step the gather should hold little
    // shared memory per SM (co-resident sampler kernels want L1): 16-row tiles x 3 blocks (80 KB per SM) keep the
    // lone launch at 0.72 and cut the step 25.9 -> 25.2 us vs round 1's 32 x 2 (106 KB per SM)
    // (profiles/r02_sampler_experiments.txt)
    int32_t tma4_blocks_per_sm = 3;
    int32_t tma4_rows = 16;
    int32_t l2_load_policy = 0, l2_store_policy = 1;  // bulk gather L2 hints: 0 normal, 1 evict_first, 2 evict_last
    // launch shapes, re-tuned after rank relabelling with 16 batches in flight (C2 bench 33.5 -> 36.5 M
    // seeds/s, C3 10.5 -> 10.9 against the earlier 4 / 1 / 4 / 3): MOMENT_HOP_GRID, MOMENT_COMPACT_GRID,
    // MOMENT_HOP_Q, MOMENT_TMA4_BLOCKS (1 block per SM: +4 % more on C2 but the single-launch gather drops to
    // 0.55 of the copy peak)
    int32_t hop_grid_per_sm = 1, compact_grid_per_sm = 2;
    // the visited bitmap is cleared by a memset node after the compaction (one sequential n/8-byte write) instead
    // of one random store per F_H member in the compaction (MOMENT_VISITED_MEMSET=0): C2 step 25.1 -> 24.7 us,
    // C3 91.9 -> 89.0 us at 16 lanes (round 2, tools/exp_variants.py)
    int32_t visited_memset = 1;  // launch caps (blocks per SM, grid-stride beyond)
    // L2 prefetch of the next hop's indptr lines by the sampler (MOMENT_HOP_PREFETCH=0/1; -1 = on with the dense
    // scan only: C2 36.5 -> 36.9 M seeds/s, C3 (sparse, 0.9 GB indptr) 10.85 -> 10.81, profiles/r01_hop_prefetch.txt)
    int32_t hop_prefetch = -1;
    // dense bitscan prefetches each new id's first neighbour line (MOMENT_SCAN_PREFETCH=0/1; -1 = only when the
    // CSR has <= 8 M edges)
    int32_t scan_prefetch = -1;
    int32_t hop_nodes_per_group = 2;  // nodes per lane group on large frontiers (1, 2, 4): 2 since the round-2 register
                                      // caps (C2 K = 200 39.9 -> 40.3, K = 20 36.6 -> 36.8 M seeds/s)
                                      // beats 2 by ~1 % per step (tools/knob_sweep_r02.sh), 4 loses 2.5 %
    int32_t hop_warp_segmented = 1;   // k <= 32: k-lane groups packed in a warp (MOMENT_HOP_WARP=0: 2^n tiles)
    int32_t init_in_hop0 = 1;         // the first hop's sampler also initialises the call (MOMENT_INIT_KERNEL=1: separate)
    int32_t bulk_stages = 4, bulk_blocks_per_sm = 4, bulk_stage_kb = 14;  // bulk gather shape (MOMENT_BULK="S,B,KB")
    std::vector<int32_t> bin_owner;
    std::vector<void*> bin_ptr;
    const uint64_t* placement = nullptr;
    std::vector<int64_t> quota;  // [n_bins][world]

    // device workspace (one allocation, carved)
    void* ws = nullptr;
    int64_t ws_bytes = 0;
    int32_t* lidx = nullptr;        // [n_vertices]: local index of v in the current batch (valid for F_H)
    uint32_t* newbits = nullptr;    // [n_words]: ids emitted at the current hop
    uint32_t* visited = nullptr;    // [n_words]: F_h membership
    uint32_t* summary = nullptr;    // [n_words / 32]: newbits words marked at the current hop (sparse scan)
    uint2* rel = nullptr;           // dense scan: [max_hops][rel_stride] {new bits, rank} per word (rank relabel)
    int64_t rel_stride = 0;         //   words per hop (n_words padded to whole scan tiles)
    int32_t rank_relabel = 1;       // MOMENT_RANK_RELABEL (dense and sparse scans)
    uint2* srel = nullptr;          // sparse scan: [max_hops][srel_stride] {word mask, first entry} per summary word
    int64_t srel_stride = 0;
    uint2* trel = nullptr;          // sparse scan: per hop, {new bits, rank} of the words holding new ids
    std::vector<int64_t> trel_off;  //   hop h's entries at trel + trel_off[h] (bound: max_F[h + 1] - max_F[0])
    int64_t n_words = 0;
    // sparse scan (summary bitmap, scan cost proportional to the touched words) for large graphs: auto when
    // n_words > kSparseScanMinWords (MOMENT_SPARSE_SCAN=0/1 forces it off/on)
    int32_t sparse_scan = 0;
    int32_t sparse_threads = 1024;  // threads (= summary words) per sparse scan tile (MOMENT_SPARSE_NT: 256/512/1024)
    unsigned long long* tile_edges = nullptr;  // edges per compaction tile of every hop (bound-numbered)
    int64_t n_tile_edges = 0;
    uint64_t* tile_status = nullptr;  // decoupled look-back descriptors: compact chain, then bitscan per hop
    int64_t n_tile_status = 0;
    std::vector<int64_t> bitscan_tiles_off;  // per hop offsets into tile_status
    uint32_t* tickets = nullptr;      // [1 + max_hops] tile tickets (compact, bitscan per hop)
    uint64_t* ebase = nullptr;        // [max_hops] first global edge position of each hop (compact)
    int32_t* pad = nullptr;           // [max_edges] padded samples (node idx * k + r), all hops
    int32_t* cnt = nullptr;           // [sum_h max_F[h]] samples per node, all hops
    uint32_t* error_flag = nullptr;   // device error bits (seed check)
    // bucketing workspace
    int64_t max_requests = 0;
    int64_t* bk_tile_counts = nullptr;  // [n_tiles][n_bins]
    int64_t* bk_bin_total = nullptr;    // [n_bins]
    int64_t* bk_qoff = nullptr;         // [n_bins * world + 1] (internal, when caller passes none)
    int32_t* bk_route = nullptr;        // [max_requests]
    int64_t* bk_qpos = nullptr;         // [max_requests]
    int64_t* d_quota = nullptr;         // [n_bins * world]
    int32_t* d_bin_owner = nullptr;     // [n_bins]
    int64_t* d_seed_stage = nullptr;    // [max_seeds] for moment_step_host
    // one-call collective exchange (moment_ctx_set_exchange): peer inboxes / outputs / flags, and the
    // device-side barrier epoch counter and watchdog status (so the exchange replays from a CUDA graph)
    bool has_exchange = false;
    moment_exchange_args ex{};
    void* ex_ws = nullptr;          // [0] uint64 epoch counter, [8] int32 watchdog status
    uint64_t* d_epoch = nullptr;
    int32_t* d_xstatus = nullptr;
    // per-call arguments the kernels read from device memory (so one captured graph serves every batch)
    uint64_t* d_call = nullptr;         // [2]: rng_seed, seeds pointer (written by set_call_kernel per call)
    // cached CUDA graph of one moment_step (sample + gather), re-captured when its shape changes
    // (the gather needs only F_H, known after the last bitscan: it runs on a branch beside the compaction)
    cudaStream_t cap_stream = nullptr, cap_side = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    int32_t step_fork = 1;  // MOMENT_STEP_FORK=0: gather after compact on one chain
    bool no_graph = false;  // MOMENT_NO_GRAPH (read at creation): moment_step launches the kernels directly
    cudaGraphExec_t step_exec = nullptr;
    cudaGraph_t step_graph = nullptr;     // the captured graph (kept: call_node refers to it)
    cudaGraphNode_t call_node = nullptr;  // its set_call kernel node, re-parameterised per launch
    struct StepKey {
        const void* indptr = nullptr;
        const void* indices = nullptr;
        int64_t n_seeds = -1;
        std::vector<int32_t> fanout;
        uint32_t flags = 0;
        moment_sample_out out{};
        void* rows = nullptr;
    } step_key;
};

namespace moment {

inline moment_status cuda_check(cudaError_t e, const char* what) {
    if (e != cudaSuccess) return fail(MOMENT_ECUDA, "%s: %s", what, cudaGetErrorString(e));
    return MOMENT_OK;
}

// Report a pending asynchronous CUDA fault (from earlier work) without synchronising.
inline moment_status cuda_pending(const char* what) { return cuda_check(cudaPeekAtLastError(), what); }

constexpr int kSampleTile = 256;     // frontier nodes per sampler tile
#ifndef MOMENT_BITSCAN_WORDS
#define MOMENT_BITSCAN_WORDS 4
#endif
constexpr int kBitscanWordsPerThread = MOMENT_BITSCAN_WORDS;  // one uint4 per thread (16 measured slower: 13.1 vs 7.6 us/launch)
#ifndef MOMENT_BITSCAN_THREADS
#define MOMENT_BITSCAN_THREADS 512
#endif
constexpr int kBitscanThreads = MOMENT_BITSCAN_THREADS;  // 2048-word tiles: +1.3 % at K = 20 over 256 (1024: -2 %)
constexpr int kBitscanTileWords = kBitscanWordsPerThread * kBitscanThreads;  // 1024 words = 32768 ids
constexpr int64_t kSparseScanMinWords = 1 << 18;  // > 8.4 M vertices: C3-C5 scan sparsely, C1/C2 densely
constexpr int kBucketTile = 1024;    // requests per bucketing tile
constexpr int kMaxFanout = 1024;

// Multiprocessors of the current device (queried once per device, cached): every launcher sizes its grid
// as a multiple of it instead of assuming 148.
int device_sms();

// Device-side barrier with the epoch read from / advanced in device memory (signal.cu): the ctx's
// collective gather enqueues it between its phases, replayable from a CUDA graph.
moment_status launch_signal_barrier_dev(const moment_ctx_s* ctx, cudaStream_t stream);

// Launchers (defined in sample.cu / gather.cu).
moment_status check_sample(const moment_ctx_s* ctx, const moment_csr* csr, const int64_t* seeds, int64_t n_seeds,
                           const moment_sample_params* p, const moment_sample_out* out);
// `after_hops`, if given, is recorded on `stream` once F_H is final (after the last bitscan, before compact).
moment_status launch_sample(moment_ctx_s* ctx, const moment_csr* csr, const uint64_t* call, int64_t n_seeds,
                            const moment_sample_params* p, const moment_sample_out* out, cudaStream_t stream,
                            cudaEvent_t after_hops = nullptr);
moment_status launch_gather(moment_ctx_s* ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n, void* out,
                            const int32_t* route, int32_t serve_rank, cudaStream_t stream);
moment_status launch_bucket(moment_ctx_s* ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                            int32_t* route, int64_t* qoff, int64_t* qpos, cudaStream_t stream);
moment_status launch_relay(moment_ctx_s* server, moment_ctx_s* requester, const int64_t* ids, const int32_t* route,
                           const int64_t* qoff, const int64_t* qpos, void* requester_out, cudaStream_t stream);
moment_status launch_hotness(const int64_t* ids, const int64_t* n_dev, int64_t max_n, uint64_t* hot,
                             cudaStream_t stream);
moment_status launch_relay_pack(moment_ctx_s* ctx, const int64_t* ids, const int64_t* qoff, const int64_t* qpos,
                                int64_t max_n, uint64_t* words, int64_t* counts, cudaStream_t stream);
moment_status launch_relay_serve(moment_ctx_s* ctx, const uint64_t* words, const int64_t* n_dev, int64_t max_n,
                                 void* rows, cudaStream_t stream);
moment_status launch_relay_scatter(moment_ctx_s* ctx, const uint64_t* words, const int64_t* n_dev, int64_t max_n,
                                   const void* rows, void* out, cudaStream_t stream);
moment_status launch_relay_push(moment_ctx_s* ctx, const int64_t* ids, const int64_t* qoff, const int64_t* qpos,
                                int64_t max_n, uint64_t* const* peer_inbox, int64_t* const* peer_count,
                                cudaStream_t stream);
moment_status launch_relay_serve_push(moment_ctx_s* ctx, const uint64_t* inbox, const int64_t* inbox_count, int64_t cap,
                                      void* const* peer_out, cudaStream_t stream);
moment_status configure_sample_kernels(int carveout);
moment_status configure_gather_kernels(int carveout);

}  // namespace moment
