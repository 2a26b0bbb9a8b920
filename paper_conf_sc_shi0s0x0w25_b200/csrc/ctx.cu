// ctx.cu — device context (workspace sized once, no allocation on the hot path) and the device entry
// points of include/moment.h: moment_sample, moment_gather, moment_gather_group, moment_bucket,
// moment_hotness, moment_step_host.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <string>
#include <cstring>
#include <mutex>
#include <new>

#include "ctx.h"

using namespace moment;

namespace {

struct Carver {
    int64_t off = 0;
    template <typename T>
    int64_t take(int64_t count) {
        off = (off + 255) & ~int64_t(255);
        int64_t at = off;
        off += std::max<int64_t>(count, 1) * (int64_t)sizeof(T);
        return at;
    }
};

moment_status check_ctx(moment_ctx_t ctx, const char* what) {
    if (!ctx) return fail(MOMENT_EINVAL, "%s: null ctx", what);
    int dev = -1;
    MOMENT_TRY(cuda_check(cudaGetDevice(&dev), what));
    if (dev != ctx->device) return fail(MOMENT_EINVAL, "%s: current device %d is not the ctx device %d", what, dev, ctx->device);
    return MOMENT_OK;
}

bool has_remote_relay(const moment_ctx_s* c);

// The per-batch exchange of one process per GPU as one enqueue (moment_ctx_set_exchange): bucket, this
// rank's own reads, requests pushed into the relays' inboxes, barrier, relayed rows pushed into the
// requesters' outputs, barrier. Every buffer is the ctx's (bucketing workspace) or registered with it.
moment_status launch_gather_collective(moment_ctx_s* c, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                                       void* out, cudaStream_t s) {
    MOMENT_TRY(launch_bucket(c, ids, n_dev, max_n, c->bk_route, c->bk_qoff, c->bk_qpos, s));
    MOMENT_TRY(launch_gather(c, ids, n_dev, max_n, out, c->bk_route, c->rank, s));
    MOMENT_TRY(launch_relay_push(c, ids, c->bk_qoff, c->bk_qpos, max_n, c->ex.peer_inbox, c->ex.peer_count, s));
    MOMENT_TRY(launch_signal_barrier_dev(c, s));  // every rank's requests are in its relays' inboxes
    MOMENT_TRY(launch_relay_serve_push(c, c->ex.inbox, c->ex.inbox_count, c->ex.cap, c->ex.peer_out, s));
    return launch_signal_barrier_dev(c, s);       // every relayed row is in its requester's output
}

// Gather for moment_gather / moment_step: the collective exchange when the quota relays rows through other
// ranks (checked by check_gather_out), else the direct gather.
moment_status launch_gather_any(moment_ctx_s* c, const int64_t* ids, const int64_t* n_dev, int64_t max_n, void* out,
                                cudaStream_t s) {
    if (c->world > 1 && c->has_exchange && has_remote_relay(c))
        return launch_gather_collective(c, ids, n_dev, max_n, out, s);
    return launch_gather(c, ids, n_dev, max_n, out, nullptr, c->rank, s);
}

// A gather whose quota relays through other ranks needs the registered exchange and its output buffer.
moment_status check_gather_out(const moment_ctx_s* c, const void* out, int64_t max_n, const char* what) {
    if (c->world > 1 && has_remote_relay(c)) {
        if (!c->has_exchange)
            return fail(MOMENT_EUNSUPPORTED, "%s: the quota relays host rows through other ranks: call "
                        "moment_ctx_set_exchange first (or use moment_gather_group)", what);
        if (out != c->ex.out)
            return fail(MOMENT_EINVAL, "%s: with relays through other ranks the output must be the registered "
                        "exchange output", what);
        if (max_n > c->ex.cap || max_n > c->max_requests)
            return fail(MOMENT_EOVERFLOW, "%s: max_n %lld > exchange cap %lld / workspace %lld", what, (long long)max_n,
                        (long long)c->ex.cap, (long long)c->max_requests);
    }
    return MOMENT_OK;
}

bool has_remote_relay(const moment_ctx_s* c) {
    for (int b = 0; b < c->n_bins; b++) {
        if (c->bin_owner[b] >= 0 || c->quota.empty()) continue;
        for (int h = 0; h < c->world; h++)
            if (h != c->rank && c->quota[(size_t)b * c->world + h] > 0) return true;
    }
    return false;
}

}  // namespace

int moment::device_sms() {
    static int cache[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0) return 148;
    if (dev < 64 && cache[dev] > 0) return cache[dev];
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
    if (dev < 64) cache[dev] = n;
    return n;
}

extern "C" moment_status moment_ctx_create(const moment_ctx_args* a, moment_ctx_t* out) {
    if (!a || !out) return fail(MOMENT_EINVAL, "moment_ctx_create: null argument");
    *out = nullptr;
    if (a->world < 1 || a->rank < 0 || a->rank >= a->world || a->world > 64)
        return fail(MOMENT_EINVAL, "moment_ctx_create: rank %d / world %d invalid", a->rank, a->world);
    if (a->n_vertices <= 0 || a->n_vertices >= (int64_t(1) << 31))
        return fail(MOMENT_EINVAL, "moment_ctx_create: n_vertices %lld must be in [1, 2^31)", (long long)a->n_vertices);
    if (a->max_seeds < 0 || a->max_hops < 0 || a->max_hops > 16 || (a->max_hops > 0 && !a->max_fanout))
        return fail(MOMENT_EINVAL, "moment_ctx_create: bad max_seeds / max_hops / max_fanout");
    if (a->n_bins < 0 || a->n_bins > MOMENT_MAX_BINS) return fail(MOMENT_EINVAL, "moment_ctx_create: n_bins %d", a->n_bins);
    if (a->n_bins > 0) {
        if (a->row_bytes <= 0 || a->row_bytes % 16 || a->row_stride < a->row_bytes || a->row_stride % 16)
            return fail(MOMENT_EINVAL, "moment_ctx_create: row_bytes %lld / row_stride %lld must be positive multiples of 16",
                        (long long)a->row_bytes, (long long)a->row_stride);
        if (!a->bin_ptr || !a->bin_owner) return fail(MOMENT_EINVAL, "moment_ctx_create: bin_ptr / bin_owner null");
        for (int b = 0; b < a->n_bins; b++) {
            if (!a->bin_ptr[b] || (reinterpret_cast<uintptr_t>(a->bin_ptr[b]) & 15))
                return fail(MOMENT_EINVAL, "moment_ctx_create: bin %d pointer null or not 16-byte aligned", b);
            if (a->bin_owner[b] < -1 || a->bin_owner[b] >= a->world)
                return fail(MOMENT_EINVAL, "moment_ctx_create: bin %d owner %d", b, a->bin_owner[b]);
        }
        if (!a->placement && a->n_bins != 1)
            return fail(MOMENT_EINVAL, "moment_ctx_create: a NULL placement means one replicated bin");
        if (a->quota)
            for (int64_t i = 0; i < (int64_t)a->n_bins * a->world; i++)
                if (a->quota[i] < 0) return fail(MOMENT_EINVAL, "moment_ctx_create: negative quota");
    }
    for (int h = 0; h < a->max_hops; h++)
        if (a->max_fanout[h] < 1 || a->max_fanout[h] > kMaxFanout)
            return fail(MOMENT_EINVAL, "moment_ctx_create: max_fanout[%d] = %d outside [1, %d]", h, a->max_fanout[h], kMaxFanout);
    int cur = -1;
    MOMENT_TRY(cuda_check(cudaGetDevice(&cur), "moment_ctx_create"));
    if (cur != a->device) MOMENT_TRY(cuda_check(cudaSetDevice(a->device), "moment_ctx_create: set device"));

    auto* c = new (std::nothrow) moment_ctx_s;
    if (!c) return fail(MOMENT_ENOMEM, "moment_ctx_create: out of host memory");
    c->rank = a->rank;
    c->world = a->world;
    c->device = a->device;
    c->n_vertices = a->n_vertices;
    c->max_seeds = a->max_seeds;
    c->max_hops = a->max_hops;
    c->max_fanout.assign(a->max_fanout, a->max_fanout + a->max_hops);
    c->row_bytes = a->row_bytes;
    c->row_stride = a->row_stride;
    c->n_bins = a->n_bins;
    c->bin_owner.assign(a->bin_owner, a->bin_owner + a->n_bins);
    c->bin_ptr.assign(a->bin_ptr, a->bin_ptr + a->n_bins);
    c->placement = a->placement;
    device_sms();  // query (and cache) the device's multiprocessor count once, outside any stream capture
    if (const char* gp = std::getenv("MOMENT_GATHER_PATH")) {
        const std::string v(gp);
        c->gather_path = v == "ldg" ? 1 : (v == "bulk" ? 2 : (v == "tma4" ? 3 : 0));
    }
    if (const char* v = std::getenv("MOMENT_TMA_PROMO")) c->tma_promo = std::max(0, std::min(3, std::atoi(v)));
    if (const char* v = std::getenv("MOMENT_TMA4_BLOCKS")) c->tma4_blocks_per_sm = std::max(1, std::atoi(v));
    if (const char* v = std::getenv("MOMENT_TMA4_ROWS")) c->tma4_rows = std::atoi(v);
    if (const char* v = std::getenv("MOMENT_BULK"))
        std::sscanf(v, "%d,%d,%d", &c->bulk_stages, &c->bulk_blocks_per_sm, &c->bulk_stage_kb);
    if (const char* v = std::getenv("MOMENT_HOP_GRID")) c->hop_grid_per_sm = std::max(1, std::atoi(v));
    if (const char* v = std::getenv("MOMENT_HOP_PREFETCH")) c->hop_prefetch = std::atoi(v);
    if (const char* v = std::getenv("MOMENT_SCAN_PREFETCH")) c->scan_prefetch = std::atoi(v);
    if (const char* v = std::getenv("MOMENT_HOP_Q")) c->hop_nodes_per_group = std::max(1, std::atoi(v));
    if (const char* v = std::getenv("MOMENT_HOP_WARP")) c->hop_warp_segmented = std::atoi(v) != 0;
    if (const char* v = std::getenv("MOMENT_STEP_FORK")) c->step_fork = std::atoi(v) != 0;
    c->no_graph = std::getenv("MOMENT_NO_GRAPH") != nullptr;
    if (const char* v = std::getenv("MOMENT_INIT_KERNEL")) c->init_in_hop0 = std::atoi(v) == 0;
    if (const char* v = std::getenv("MOMENT_VISITED_MEMSET")) c->visited_memset = std::atoi(v);
    if (const char* v = std::getenv("MOMENT_COMPACT_GRID")) c->compact_grid_per_sm = std::max(1, std::atoi(v));
    c->sparse_scan = (a->n_vertices + 31) / 32 > kSparseScanMinWords;
    if (const char* v = std::getenv("MOMENT_SPARSE_SCAN")) c->sparse_scan = std::atoi(v) != 0;
    if (const char* v = std::getenv("MOMENT_RANK_RELABEL")) c->rank_relabel = std::atoi(v) != 0;
    if (const char* v = std::getenv("MOMENT_SPARSE_NT")) {
        const int nt = std::atoi(v);
        c->sparse_threads = nt >= 1024 ? 1024 : nt >= 512 ? 512 : 256;
    }
    if (const char* l2 = std::getenv("MOMENT_GATHER_L2")) {  // "<load><store>" digits, e.g. "01"
        if (std::strlen(l2) == 2) {
            c->l2_load_policy = l2[0] - '0';
            c->l2_store_policy = l2[1] - '0';
        }
    }
    if (a->quota) c->quota.assign(a->quota, a->quota + (size_t)a->n_bins * a->world);
    // bounds per hop
    c->max_F.resize(a->max_hops + 1);
    c->max_E.resize(a->max_hops);
    int64_t F = std::min(a->max_seeds, a->n_vertices);
    c->max_F[0] = F;
    for (int h = 0; h < a->max_hops; h++) {
        c->max_E[h] = F * a->max_fanout[h];
        c->max_edges += c->max_E[h];
        c->max_offsets += F + 1;
        F = std::min(F + F * (int64_t)a->max_fanout[h], a->n_vertices);
        c->max_F[h + 1] = F;
    }
    c->max_nodes = std::max<int64_t>(F, a->max_seeds);
    c->n_words = (a->n_vertices + 31) / 32;
    c->max_requests = c->max_nodes;
    // carve the workspace
    Carver cv;
    const int64_t o_lidx = cv.take<int32_t>(a->n_vertices);
    const int64_t n_words_pad = (c->n_words + kBitscanTileWords - 1) / kBitscanTileWords * kBitscanTileWords;
    const int64_t o_newbits = cv.take<uint32_t>(n_words_pad);
    const int64_t o_visited = cv.take<uint32_t>(n_words_pad);
    const int64_t o_summary = cv.take<uint32_t>(n_words_pad / 32);
    // rank relabelling (dense scan): per hop {new bits, rank} of every bitmap word, L2-resident (C2: 612 KB
    // per hop) instead of random lidx traffic over n int32 (C2: 9.8 MB per ctx)
    const bool rel_on = !c->sparse_scan && c->rank_relabel && a->max_hops > 0;
    const int64_t o_rel = rel_on ? cv.take<uint2>(n_words_pad * a->max_hops) : -1;
    // sparse scan: two-level tables (summary-word level + one entry per word holding new ids); entries of
    // hop h <= min(its new ids, words) <= min(max_F[h] * max_fanout[h], n_words)
    const bool srel_on = c->sparse_scan && c->rank_relabel && a->max_hops > 0;
    const int64_t n_summary_pad = n_words_pad / 32;
    const int64_t o_srel = srel_on ? cv.take<uint2>(n_summary_pad * a->max_hops) : -1;
    c->trel_off.assign(a->max_hops + 1, 0);
    for (int h = 0; h < a->max_hops; h++)
        c->trel_off[h + 1] = c->trel_off[h] + std::max<int64_t>(1, std::min<int64_t>(c->max_F[h] * a->max_fanout[h],
                                                                                        n_words_pad));
    const int64_t o_trel = srel_on ? cv.take<uint2>(c->trel_off[a->max_hops]) : -1;
    const int64_t scan_tiles = n_words_pad / kBitscanTileWords;
    c->bitscan_tiles_off.resize(a->max_hops);
    int64_t nts = 0, cnt_total = 0;
    for (int h = 0; h < a->max_hops; h++) {  // compact chain: hop-aligned tiles of all hops
        nts += (c->max_F[h] + kSampleTile - 1) / kSampleTile;
        cnt_total += c->max_F[h];
    }
    for (int h = 0; h < a->max_hops; h++) {
        c->bitscan_tiles_off[h] = nts;
        nts += scan_tiles;
    }
    c->n_tile_status = std::max<int64_t>(nts, 1);
    const int64_t o_tiles = cv.take<uint64_t>(c->n_tile_status);
    c->n_tile_edges = 0;
    for (int h = 0; h < a->max_hops; h++) c->n_tile_edges += (c->max_F[h] + kSampleTile - 1) / kSampleTile;
    const int64_t o_tile_edges = cv.take<unsigned long long>(std::max<int64_t>(c->n_tile_edges, 1));
    const int64_t o_tickets = cv.take<uint32_t>(1 + std::max(1, a->max_hops));
    const int64_t o_ebase = cv.take<uint64_t>(std::max(1, a->max_hops));
    const int64_t o_pad = cv.take<int32_t>(c->max_edges);
    const int64_t o_cnt = cv.take<int32_t>(cnt_total);
    const int64_t o_err = cv.take<uint32_t>(1);
    const int32_t Q = std::max(1, a->n_bins * a->world);
    const int64_t bk_tiles = (c->max_requests + kBucketTile - 1) / kBucketTile + 1;
    int64_t o_bk_tc = 0, o_bk_tot = 0, o_bk_qoff = 0, o_bk_route = 0, o_bk_qpos = 0, o_quota = 0, o_owner = 0;
    if (a->n_bins > 0) {
        o_bk_tc = cv.take<int64_t>(bk_tiles * std::max<int64_t>(Q, a->n_bins));
        o_bk_tot = cv.take<int64_t>(a->n_bins);
        o_bk_qoff = cv.take<int64_t>(Q + 1);
        o_bk_route = cv.take<int32_t>(c->max_requests);
        o_bk_qpos = cv.take<int64_t>(c->max_requests);
        o_quota = cv.take<int64_t>(Q);
        o_owner = cv.take<int32_t>(a->n_bins);
    }
    const int64_t o_seed = cv.take<int64_t>(a->max_seeds);
    const int64_t o_call = cv.take<uint64_t>(3);
    c->ws_bytes = cv.off;
    cudaError_t e = cudaMalloc(&c->ws, c->ws_bytes);
    if (e != cudaSuccess) {
        delete c;
        return fail(MOMENT_ENOMEM, "moment_ctx_create: cudaMalloc(%lld bytes): %s", (long long)cv.off, cudaGetErrorString(e));
    }
    char* w = static_cast<char*>(c->ws);
    c->lidx = reinterpret_cast<int32_t*>(w + o_lidx);
    c->newbits = reinterpret_cast<uint32_t*>(w + o_newbits);
    c->visited = reinterpret_cast<uint32_t*>(w + o_visited);
    c->summary = reinterpret_cast<uint32_t*>(w + o_summary);
    c->rel = rel_on ? reinterpret_cast<uint2*>(w + o_rel) : nullptr;
    c->rel_stride = n_words_pad;
    c->srel = srel_on ? reinterpret_cast<uint2*>(w + o_srel) : nullptr;
    c->srel_stride = n_summary_pad;
    c->trel = srel_on ? reinterpret_cast<uint2*>(w + o_trel) : nullptr;
    c->tile_status = reinterpret_cast<uint64_t*>(w + o_tiles);
    c->tile_edges = reinterpret_cast<unsigned long long*>(w + o_tile_edges);
    c->tickets = reinterpret_cast<uint32_t*>(w + o_tickets);
    c->ebase = reinterpret_cast<uint64_t*>(w + o_ebase);
    c->pad = reinterpret_cast<int32_t*>(w + o_pad);
    c->cnt = reinterpret_cast<int32_t*>(w + o_cnt);
    c->error_flag = reinterpret_cast<uint32_t*>(w + o_err);
    if (a->n_bins > 0) {
        c->bk_tile_counts = reinterpret_cast<int64_t*>(w + o_bk_tc);
        c->bk_bin_total = reinterpret_cast<int64_t*>(w + o_bk_tot);
        c->bk_qoff = reinterpret_cast<int64_t*>(w + o_bk_qoff);
        c->bk_route = reinterpret_cast<int32_t*>(w + o_bk_route);
        c->bk_qpos = reinterpret_cast<int64_t*>(w + o_bk_qpos);
        c->d_quota = reinterpret_cast<int64_t*>(w + o_quota);
        c->d_bin_owner = reinterpret_cast<int32_t*>(w + o_owner);
    }
    c->d_seed_stage = reinterpret_cast<int64_t*>(w + o_seed);
    c->d_call = reinterpret_cast<uint64_t*>(w + o_call);
    moment_status st = MOMENT_OK;
    do {
        {  // kernel attributes, once per device. Shared-memory carveout preference (percent of the unified
           // L1 / shared storage): the sampler kernels ask for 25 % (L1 for their random CSR / rank-table reads:
           // +2.4 % at K = 20, +0.4 % at K = 200; 0 % forces reconfigurations, 100 % starves compact of L1, 2x
           // slower), the gathers keep the driver's per-kernel choice (-1). MOMENT_CARVEOUT sets both,
           // MOMENT_CARVEOUT_SAMPLE / _GATHER one group (tools/sweep_carveout.sh)
            static std::mutex mu;
            static uint64_t done = 0;
            std::lock_guard<std::mutex> lock(mu);
            if (a->device < 64 && !(done >> a->device & 1)) {
                const char* cv_env = std::getenv("MOMENT_CARVEOUT");
                int carve_s = cv_env ? std::atoi(cv_env) : 25, carve_g = cv_env ? std::atoi(cv_env) : -1;
                if (const char* v = std::getenv("MOMENT_CARVEOUT_SAMPLE")) carve_s = std::atoi(v);
                if (const char* v = std::getenv("MOMENT_CARVEOUT_GATHER")) carve_g = std::atoi(v);
                if ((st = configure_sample_kernels(carve_s)) != MOMENT_OK) break;
                if ((st = configure_gather_kernels(carve_g)) != MOMENT_OK) break;
                done |= 1ull << a->device;
            }
        }
        if ((st = cuda_check(cudaStreamCreateWithFlags(&c->cap_stream, cudaStreamNonBlocking), "moment_ctx_create: stream")) != MOMENT_OK) break;
        if ((st = cuda_check(cudaStreamCreateWithFlags(&c->cap_side, cudaStreamNonBlocking), "moment_ctx_create: stream")) != MOMENT_OK) break;
        if ((st = cuda_check(cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming), "moment_ctx_create: event")) != MOMENT_OK) break;
        if ((st = cuda_check(cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming), "moment_ctx_create: event")) != MOMENT_OK) break;
        if ((st = cuda_check(cudaMemset(c->ws, 0, c->ws_bytes), "moment_ctx_create: memset")) != MOMENT_OK) break;
        if ((st = cuda_check(cudaMemset(c->lidx, 0xFF, a->n_vertices * sizeof(int32_t)), "moment_ctx_create: memset")) != MOMENT_OK) break;
        if (a->n_bins > 0) {
            std::vector<int64_t> q((size_t)Q, 0);
            if (!c->quota.empty()) std::copy(c->quota.begin(), c->quota.end(), q.begin());
            if ((st = cuda_check(cudaMemcpy(c->d_quota, q.data(), Q * sizeof(int64_t), cudaMemcpyHostToDevice), "quota")) != MOMENT_OK) break;
            if ((st = cuda_check(cudaMemcpy(c->d_bin_owner, c->bin_owner.data(), a->n_bins * sizeof(int32_t), cudaMemcpyHostToDevice), "owner")) != MOMENT_OK) break;
        }
        st = cuda_check(cudaDeviceSynchronize(), "moment_ctx_create: sync");
    } while (0);
    if (cur != a->device) cudaSetDevice(cur);
    if (st != MOMENT_OK) {
        moment_ctx_free(c);
        return st;
    }
    *out = c;
    return MOMENT_OK;
}

extern "C" moment_status moment_ctx_free(moment_ctx_t ctx) {
    if (!ctx) return MOMENT_OK;
    int cur = -1;
    cudaGetDevice(&cur);
    cudaSetDevice(ctx->device);
    if (ctx->step_exec) cudaGraphExecDestroy(ctx->step_exec);
    if (ctx->step_graph) cudaGraphDestroy(ctx->step_graph);
    if (ctx->cap_stream) cudaStreamDestroy(ctx->cap_stream);
    if (ctx->cap_side) cudaStreamDestroy(ctx->cap_side);
    if (ctx->ev_fork) cudaEventDestroy(ctx->ev_fork);
    if (ctx->ev_join) cudaEventDestroy(ctx->ev_join);
    cudaError_t e = ctx->ws ? cudaFree(ctx->ws) : cudaSuccess;
    if (ctx->ex_ws) cudaFree(ctx->ex_ws);
    cudaSetDevice(cur);
    delete ctx;
    return cuda_check(e, "moment_ctx_free");
}

extern "C" moment_status moment_ctx_set_exchange(moment_ctx_t ctx, const moment_exchange_args* a) {
    MOMENT_TRY(check_ctx(ctx, "moment_ctx_set_exchange"));
    if (!a) return fail(MOMENT_EINVAL, "moment_ctx_set_exchange: null argument");
    if (ctx->world > MOMENT_MAX_WORLD) return fail(MOMENT_EUNSUPPORTED, "moment_ctx_set_exchange: world > %d", MOMENT_MAX_WORLD);
    if (a->cap < 0 || a->timeout_ns <= 0) return fail(MOMENT_EINVAL, "moment_ctx_set_exchange: cap < 0 or timeout <= 0");
    if (!a->inbox || !a->inbox_count || !a->flags || !a->out || (reinterpret_cast<uintptr_t>(a->out) & 15))
        return fail(MOMENT_EINVAL, "moment_ctx_set_exchange: inbox / counts / flags / out null or out not 16-byte aligned");
    if (ctx->n_bins <= 0 || !ctx->placement) return fail(MOMENT_EINVAL, "moment_ctx_set_exchange: ctx has no placement map");
    for (int h = 0; h < ctx->world; h++) {
        if (h == ctx->rank) continue;
        if (!a->peer_inbox[h] || !a->peer_count[h] || !a->peer_flag[h] || !a->peer_out[h] ||
            (reinterpret_cast<uintptr_t>(a->peer_out[h]) & 15))
            return fail(MOMENT_EINVAL, "moment_ctx_set_exchange: peer %d pointer null or misaligned", h);
    }
    if (!ctx->ex_ws) {
        MOMENT_TRY(cuda_check(cudaMalloc(&ctx->ex_ws, 16), "moment_ctx_set_exchange: cudaMalloc"));
        MOMENT_TRY(cuda_check(cudaMemset(ctx->ex_ws, 0, 16), "moment_ctx_set_exchange: memset"));
        MOMENT_TRY(cuda_check(cudaDeviceSynchronize(), "moment_ctx_set_exchange: sync"));
        ctx->d_epoch = static_cast<uint64_t*>(ctx->ex_ws);
        ctx->d_xstatus = reinterpret_cast<int32_t*>(static_cast<char*>(ctx->ex_ws) + 8);
    }
    ctx->ex = *a;
    ctx->has_exchange = true;
    if (ctx->step_exec) {  // a cached step graph captured without the exchange is stale
        cudaGraphExecDestroy(ctx->step_exec);
        ctx->step_exec = nullptr;
        cudaGraphDestroy(ctx->step_graph);
        ctx->step_graph = nullptr;
    }
    return MOMENT_OK;
}

extern "C" moment_status moment_exchange_status(moment_ctx_t ctx, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_exchange_status"));
    if (!ctx->has_exchange) return MOMENT_OK;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    int32_t st = 0;
    MOMENT_TRY(cuda_check(cudaMemcpyAsync(&st, ctx->d_xstatus, sizeof(st), cudaMemcpyDeviceToHost, s), "moment_exchange_status"));
    MOMENT_TRY(cuda_check(cudaStreamSynchronize(s), "moment_exchange_status"));
    if (st == 0) return MOMENT_OK;
    MOMENT_TRY(cuda_check(cudaMemsetAsync(ctx->d_xstatus, 0, sizeof(int32_t), s), "moment_exchange_status"));
    MOMENT_TRY(cuda_check(cudaStreamSynchronize(s), "moment_exchange_status"));
    return fail(MOMENT_ETIMEDOUT, "moment_exchange_status: a device barrier of rank %d timed out", ctx->rank);
}

extern "C" moment_status moment_ctx_workspace_bytes(moment_ctx_t ctx, int64_t* bytes) {
    if (!ctx || !bytes) return fail(MOMENT_EINVAL, "moment_ctx_workspace_bytes: null argument");
    *bytes = ctx->ws_bytes;
    return MOMENT_OK;
}

namespace {

__global__ void set_call_kernel(uint64_t* call, uint64_t rng_seed, const int64_t* seeds, int64_t* counts_host,
                                unsigned long long* zero, int64_t n_zero) {
    if (threadIdx.x == 0) {
        call[0] = rng_seed;
        call[1] = reinterpret_cast<uint64_t>(seeds);
        call[2] = reinterpret_cast<uint64_t>(counts_host);  // mapped host counts (moment_step_host) or 0
    }
    for (int64_t j = threadIdx.x; j < n_zero; j += blockDim.x) zero[j] = 0;  // hop 0's compaction tile sums
}

// Stage the per-call arguments (rng_seed, seeds pointer) into the device call block with a one-warp
// kernel whose parameters carry the values: ordered before the call's kernels on `s`, and safe inside a
// caller's stream capture (the values are baked into the captured node). It also zeroes the first hop's
// compaction tile sums (the later hops' are zeroed by the scan before them).
moment_status write_call(moment_ctx_s* c, uint64_t rng_seed, const int64_t* seeds, int64_t n_seeds, cudaStream_t s,
                         int64_t* counts_host = nullptr) {
    set_call_kernel<<<1, 32, 0, s>>>(c->d_call, rng_seed, seeds, counts_host, c->tile_edges,
                                     std::min<int64_t>((n_seeds + kSampleTile - 1) / kSampleTile, c->n_tile_edges));
    return cuda_check(cudaGetLastError(), "call block");
}

bool same_key(const moment_ctx_s::StepKey& k, const moment_csr* csr, int64_t n_seeds, const moment_sample_params* p,
              const moment_sample_out* out, void* rows) {
    if (k.indptr != csr->indptr || k.indices != csr->indices || k.n_seeds != n_seeds || k.flags != p->flags ||
        k.rows != rows || (int)k.fanout.size() != p->n_hops)
        return false;
    for (int h = 0; h < p->n_hops; h++)
        if (k.fanout[h] != p->fanout[h]) return false;
    return std::memcmp(&k.out, out, sizeof(moment_sample_out)) == 0;
}

// One sample + gather, replayed from a cached CUDA graph (captured on first use of a shape); falls back to
// direct launches while the caller's stream is itself being captured.
// The call-block kernel's parameters for one call (the graph's first node; updated per launch).
struct CallParams {
    uint64_t* call;
    uint64_t rng_seed;
    const int64_t* seeds;
    int64_t* counts_host;
    unsigned long long* zero;
    int64_t n_zero;
};

moment_status set_call_node(moment_ctx_s* c, const CallParams& cp) {
    void* args[] = {(void*)&cp.call, (void*)&cp.rng_seed, (void*)&cp.seeds, (void*)&cp.counts_host, (void*)&cp.zero,
                    (void*)&cp.n_zero};
    cudaKernelNodeParams kp{};
    kp.func = (void*)set_call_kernel;
    kp.gridDim = dim3(1);
    kp.blockDim = dim3(32);
    kp.sharedMemBytes = 0;
    kp.kernelParams = args;
    return cuda_check(cudaGraphExecKernelNodeSetParams(c->step_exec, c->call_node, &kp), "moment_step: call node");
}

// One step (moment_step / moment_step_host): the call block (rng seed, seeds pointer, host counts pointer) is
// written by set_call_kernel, then sample + gather. From a CUDA graph cached in the ctx, the call kernel is the
// graph's first node and its parameters are replaced per launch (cudaGraphExecKernelNodeSetParams), so a step
// is one graph launch with no separate kernel launch in front of it (measured: the separate launch left a
// ~5 us gap before the first hop). While the caller's stream is being captured, or with MOMENT_NO_GRAPH, the
// kernels are launched directly.
moment_status run_step(moment_ctx_s* c, const moment_csr* csr, int64_t n_seeds, const moment_sample_params* p,
                       const moment_sample_out* out, void* rows, cudaStream_t s, const int64_t* seeds,
                       int64_t* counts_host = nullptr) {
    const int H = p->n_hops;
    const CallParams cp{c->d_call, p->rng_seed, seeds, counts_host, c->tile_edges,
                        std::min<int64_t>((n_seeds + kSampleTile - 1) / kSampleTile, c->n_tile_edges)};
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    MOMENT_TRY(cuda_check(cudaStreamIsCapturing(s, &cs), "moment_step"));
    if (cs != cudaStreamCaptureStatusNone || c->no_graph) {
        MOMENT_TRY(write_call(c, p->rng_seed, seeds, n_seeds, s, counts_host));
        MOMENT_TRY(launch_sample(c, csr, c->d_call, n_seeds, p, out, s));
        if (rows) MOMENT_TRY(launch_gather_any(c, out->nodes, out->counts + H, out->cap_nodes, rows, s));
        return MOMENT_OK;
    }
    if (!c->step_exec || !same_key(c->step_key, csr, n_seeds, p, out, rows)) {
        if (c->step_exec) {
            MOMENT_TRY(cuda_check(cudaStreamSynchronize(s), "moment_step: drain before re-capture"));
            cudaGraphExecDestroy(c->step_exec);
            c->step_exec = nullptr;
        }
        if (c->step_graph) {
            cudaGraphDestroy(c->step_graph);
            c->step_graph = nullptr;
        }
        MOMENT_TRY(cuda_check(cudaStreamBeginCapture(c->cap_stream, cudaStreamCaptureModeThreadLocal), "capture"));
        const bool fork = rows && c->step_fork;
        moment_status st = write_call(c, p->rng_seed, seeds, n_seeds, c->cap_stream, counts_host);
        if (st == MOMENT_OK)
            st = launch_sample(c, csr, c->d_call, n_seeds, p, out, c->cap_stream, fork ? c->ev_fork : nullptr);
        if (st == MOMENT_OK && rows && !fork)
            st = launch_gather_any(c, out->nodes, out->counts + H, out->cap_nodes, rows, c->cap_stream);
        if (st == MOMENT_OK && fork) {  // gather on a branch that joins after the compaction
            st = cuda_check(cudaStreamWaitEvent(c->cap_side, c->ev_fork, 0), "moment_step: fork");
            if (st == MOMENT_OK)
                st = launch_gather_any(c, out->nodes, out->counts + H, out->cap_nodes, rows, c->cap_side);
            if (st == MOMENT_OK) st = cuda_check(cudaEventRecord(c->ev_join, c->cap_side), "moment_step: join");
            if (st == MOMENT_OK) st = cuda_check(cudaStreamWaitEvent(c->cap_stream, c->ev_join, 0), "moment_step: join");
        }
        cudaGraph_t g = nullptr;
        cudaError_t e = cudaStreamEndCapture(c->cap_stream, &g);
        if (st != MOMENT_OK) {
            if (g) cudaGraphDestroy(g);
            return st;
        }
        MOMENT_TRY(cuda_check(e, "moment_step: end capture"));
        // the call kernel is the graph's only root (captured first; everything else depends on it)
        size_t n_roots = 1;
        e = cudaGraphGetRootNodes(g, &c->call_node, &n_roots);
        if (e != cudaSuccess || n_roots != 1) {
            cudaGraphDestroy(g);
            return fail(MOMENT_ECUDA, "moment_step: captured graph has %zu roots", n_roots);
        }
        e = cudaGraphInstantiate(&c->step_exec, g, 0);
        if (e != cudaSuccess) {
            cudaGraphDestroy(g);
            MOMENT_TRY(cuda_check(e, "moment_step: instantiate"));
        }
        c->step_graph = g;  // kept: the call node handle refers to it
        c->step_key.indptr = csr->indptr;
        c->step_key.indices = csr->indices;
        c->step_key.n_seeds = n_seeds;
        c->step_key.fanout.assign(p->fanout, p->fanout + H);
        c->step_key.flags = p->flags;
        c->step_key.out = *out;
        c->step_key.rows = rows;
    }
    MOMENT_TRY(set_call_node(c, cp));
    return cuda_check(cudaGraphLaunch(c->step_exec, s), "moment_step: graph launch");
}

// The device address of a pinned, mapped host buffer (cudaHostAlloc / registered memory; the same address under
// unified addressing), or null for pageable memory.
template <typename T>
T* mapped_host_ptr(T* p) {
    cudaPointerAttributes a{};
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();  // pageable memory on old drivers reports an error: clear it
        return nullptr;
    }
    return a.type == cudaMemoryTypeHost && a.devicePointer ? static_cast<T*>(a.devicePointer) : nullptr;
}

moment_status check_rows(const moment_ctx_s* c, void* rows, const moment_sample_out* out) {
    if (!rows) return MOMENT_OK;
    if (c->n_bins <= 0) return fail(MOMENT_EINVAL, "moment_step: ctx has no feature bins");
    MOMENT_TRY(check_gather_out(c, rows, out->cap_nodes, "moment_step"));
    if ((reinterpret_cast<uintptr_t>(rows) & 15) != 0) return fail(MOMENT_EINVAL, "moment_step: rows must be 16-byte aligned");
    if (out->cap_nodes * (c->row_bytes / 16) >= (int64_t(1) << 32))
        return fail(MOMENT_EUNSUPPORTED, "moment_step: %lld rows exceed 2^32 vectors per call", (long long)out->cap_nodes);
    return MOMENT_OK;
}

}  // namespace

extern "C" moment_status moment_sample(moment_ctx_t ctx, const moment_csr* csr, const int64_t* seeds, int64_t n_seeds,
                                       const moment_sample_params* params, const moment_sample_out* out, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_sample"));
    MOMENT_TRY(check_sample(ctx, csr, seeds, n_seeds, params, out));
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    MOMENT_TRY(write_call(ctx, params->rng_seed, seeds, n_seeds, s));
    return launch_sample(ctx, csr, ctx->d_call, n_seeds, params, out, s);
}

extern "C" moment_status moment_step(moment_ctx_t ctx, const moment_csr* csr, const int64_t* seeds, int64_t n_seeds,
                                     const moment_sample_params* params, const moment_sample_out* out, void* d_rows,
                                     void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_step"));
    MOMENT_TRY(check_sample(ctx, csr, seeds, n_seeds, params, out));
    MOMENT_TRY(check_rows(ctx, d_rows, out));
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    return run_step(ctx, csr, n_seeds, params, out, d_rows, s, seeds);
}

extern "C" moment_status moment_step_batch(int32_t n, const moment_ctx_t* ctxs, const moment_csr* csr,
                                           const int64_t* const* seeds, int64_t n_seeds,
                                           const moment_sample_params* params, const uint64_t* rng_seeds,
                                           const moment_sample_out* outs, void* const* d_rows,
                                           int64_t* const* counts_host, void* const* streams) {
    if (n < 0 || (n > 0 && (!ctxs || !seeds || !params || !rng_seeds || !outs || !streams)))
        return fail(MOMENT_EINVAL, "moment_step_batch: null argument");
    for (int i = 0; i < n; i++)
        for (int j = 0; j < i; j++)
            if (ctxs[i] == ctxs[j]) return fail(MOMENT_EINVAL, "moment_step_batch: ctxs[%d] repeats ctxs[%d]", i, j);
    moment_sample_params p = *params;
    for (int i = 0; i < n; i++) {
        p.rng_seed = rng_seeds[i];
        void* rows = d_rows ? d_rows[i] : nullptr;
        const moment_status st =
            counts_host ? moment_step_host(ctxs[i], csr, seeds[i], n_seeds, &p, &outs[i], rows, counts_host[i], streams[i])
                        : moment_step(ctxs[i], csr, seeds[i], n_seeds, &p, &outs[i], rows, streams[i]);
        if (st != MOMENT_OK) return st;
    }
    return MOMENT_OK;
}

extern "C" moment_status moment_sample_check(moment_ctx_t ctx, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_sample_check"));
    uint32_t flag = 0;
    MOMENT_TRY(cuda_check(cudaMemcpyAsync(&flag, ctx->error_flag, sizeof(flag), cudaMemcpyDeviceToHost,
                                          static_cast<cudaStream_t>(stream)), "moment_sample_check"));
    MOMENT_TRY(cuda_check(cudaStreamSynchronize(static_cast<cudaStream_t>(stream)), "moment_sample_check"));
    MOMENT_TRY(cuda_check(cudaMemsetAsync(ctx->error_flag, 0, sizeof(uint32_t), static_cast<cudaStream_t>(stream)), "moment_sample_check"));
    if (flag & 1u) return fail(MOMENT_EINVAL, "moment_sample: a seed was out of range");
    if (flag & 2u) return fail(MOMENT_EINVAL, "moment_sample: a seed was repeated");
    return MOMENT_OK;
}

extern "C" moment_status moment_hotness(moment_ctx_t ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                                        uint64_t* hot, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_hotness"));
    if (max_n < 0 || (max_n > 0 && (!ids || !hot))) return fail(MOMENT_EINVAL, "moment_hotness: null argument");
    return launch_hotness(ids, n_dev, max_n, hot, static_cast<cudaStream_t>(stream));
}

extern "C" moment_status moment_bucket(moment_ctx_t ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                                       int32_t* route, int64_t* qoff, int64_t* qpos, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_bucket"));
    if (max_n < 0 || (max_n > 0 && (!ids || !route || !qoff || !qpos))) return fail(MOMENT_EINVAL, "moment_bucket: null argument");
    if (ctx->n_bins <= 0) return fail(MOMENT_EINVAL, "moment_bucket: ctx has no bins");
    return launch_bucket(ctx, ids, n_dev, max_n, route, qoff, qpos, static_cast<cudaStream_t>(stream));
}

extern "C" moment_status moment_gather(moment_ctx_t ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n, void* out,
                                       void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_gather"));
    MOMENT_TRY(check_gather_out(ctx, out, max_n, "moment_gather"));
    return launch_gather_any(ctx, ids, n_dev, max_n, out, static_cast<cudaStream_t>(stream));
}

extern "C" moment_status moment_gather_group(moment_ctx_t const* ctxs, int32_t world, const int64_t* const* ids,
                                             const int64_t* const* n_dev, int64_t max_n, void* const* out, void* stream) {
    if (!ctxs || !ids || !out || world < 1) return fail(MOMENT_EINVAL, "moment_gather_group: null argument");
    for (int r = 0; r < world; r++) {
        MOMENT_TRY(check_ctx(ctxs[r], "moment_gather_group"));
        if (ctxs[r]->world != world || ctxs[r]->rank != r)
            return fail(MOMENT_EINVAL, "moment_gather_group: ctxs[%d] has rank %d / world %d", r, ctxs[r]->rank, ctxs[r]->world);
        if (ctxs[r]->row_bytes != ctxs[0]->row_bytes || !ctxs[r]->placement)
            return fail(MOMENT_EINVAL, "moment_gather_group: ctxs disagree on row_bytes or lack a placement map");
        if (max_n > ctxs[r]->max_requests)
            return fail(MOMENT_EOVERFLOW, "moment_gather_group: max_n %lld > workspace %lld", (long long)max_n, (long long)ctxs[r]->max_requests);
    }
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const int64_t* nd;
    // phase 1: every rank buckets its requests (publishes its relay queues)
    for (int r = 0; r < world; r++) {
        nd = n_dev ? n_dev[r] : nullptr;
        MOMENT_TRY(launch_bucket(ctxs[r], ids[r], nd, max_n, ctxs[r]->bk_route, ctxs[r]->bk_qoff, ctxs[r]->bk_qpos, s));
    }
    // phase 2: direct reads (local / peer / host) by each requester, relays served by each relay rank
    for (int r = 0; r < world; r++) {
        nd = n_dev ? n_dev[r] : nullptr;
        MOMENT_TRY(launch_gather(ctxs[r], ids[r], nd, max_n, out[r], ctxs[r]->bk_route, r, s));
        for (int g = 0; g < world; g++) {
            if (g == r) continue;
            MOMENT_TRY(launch_relay(ctxs[r], ctxs[g], ids[g], ctxs[g]->bk_route, ctxs[g]->bk_qoff, ctxs[g]->bk_qpos, out[g], s));
        }
    }
    return MOMENT_OK;
}

extern "C" moment_status moment_step_host(moment_ctx_t ctx, const moment_csr* csr, const int64_t* seeds_host, int64_t n_seeds,
                                          const moment_sample_params* params, const moment_sample_out* out, void* d_rows,
                                          int64_t* counts_host, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_step_host"));
    if (!params || !out || !counts_host || (n_seeds > 0 && !seeds_host)) return fail(MOMENT_EINVAL, "moment_step_host: null argument");
    MOMENT_TRY(check_sample(ctx, csr, ctx->d_seed_stage, n_seeds, params, out));
    MOMENT_TRY(check_rows(ctx, d_rows, out));
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    // pinned (page-locked, device-mapped) host buffers move over PCIe inside the step's own kernels: the first
    // hop reads the seeds from host memory and the compaction's last block stores the counts there (no
    // copy-engine operation on the step's critical path); pageable buffers go through cudaMemcpyAsync
    const int64_t* seeds_dev = mapped_host_ptr(seeds_host);
    int64_t* counts_dev = mapped_host_ptr(counts_host);
    if (!seeds_dev) {
        MOMENT_TRY(cuda_check(cudaMemcpyAsync(ctx->d_seed_stage, seeds_host, n_seeds * sizeof(int64_t),
                                              cudaMemcpyHostToDevice, s), "moment_step_host: H2D"));
        seeds_dev = ctx->d_seed_stage;
    }
    MOMENT_TRY(run_step(ctx, csr, n_seeds, params, out, d_rows, s, seeds_dev, counts_dev));
    if (counts_dev) return MOMENT_OK;
    const int H = params->n_hops;
    return cuda_check(cudaMemcpyAsync(counts_host, out->counts, (2 * H + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost, s),
                      "moment_step_host: D2H");
}

// ---- H5 exchange for one process per GPU -------------------------------------------------------------
extern "C" moment_status moment_gather_routed(moment_ctx_t ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                                              const int32_t* route, void* out, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_gather_routed"));
    if (!route || !ctx->placement) return fail(MOMENT_EINVAL, "moment_gather_routed: needs a route and a placement map");
    return launch_gather(ctx, ids, n_dev, max_n, out, route, ctx->rank, static_cast<cudaStream_t>(stream));
}

extern "C" moment_status moment_relay_pack(moment_ctx_t ctx, const int64_t* ids, int64_t max_n, const int64_t* qoff,
                                           const int64_t* qpos, uint64_t* words, int64_t* send_counts, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_relay_pack"));
    if (max_n < 0 || (max_n > 0 && (!ids || !qoff || !qpos || !words)) || !send_counts)
        return fail(MOMENT_EINVAL, "moment_relay_pack: null argument");
    return launch_relay_pack(ctx, ids, qoff, qpos, max_n, words, send_counts, static_cast<cudaStream_t>(stream));
}

extern "C" moment_status moment_relay_serve(moment_ctx_t ctx, const uint64_t* words, const int64_t* n_dev, int64_t max_n,
                                            void* rows, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_relay_serve"));
    if (max_n < 0 || (max_n > 0 && (!words || !rows))) return fail(MOMENT_EINVAL, "moment_relay_serve: null argument");
    if (ctx->n_bins <= 0) return fail(MOMENT_EINVAL, "moment_relay_serve: ctx has no bins");
    return launch_relay_serve(ctx, words, n_dev, max_n, rows, static_cast<cudaStream_t>(stream));
}

extern "C" moment_status moment_relay_scatter(moment_ctx_t ctx, const uint64_t* words, const int64_t* n_dev, int64_t max_n,
                                              const void* rows, void* out, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_relay_scatter"));
    if (max_n < 0 || (max_n > 0 && (!words || !rows || !out))) return fail(MOMENT_EINVAL, "moment_relay_scatter: null argument");
    return launch_relay_scatter(ctx, words, n_dev, max_n, rows, out, static_cast<cudaStream_t>(stream));
}

extern "C" moment_status moment_relay_push(moment_ctx_t ctx, const int64_t* ids, int64_t max_n, const int64_t* qoff,
                                           const int64_t* qpos, uint64_t* const* peer_inbox, int64_t* const* peer_count,
                                           void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_relay_push"));
    if (max_n < 0 || (max_n > 0 && (!ids || !qoff || !qpos)) || !peer_inbox || !peer_count)
        return fail(MOMENT_EINVAL, "moment_relay_push: null argument");
    return launch_relay_push(ctx, ids, qoff, qpos, max_n, peer_inbox, peer_count, static_cast<cudaStream_t>(stream));
}

extern "C" moment_status moment_relay_serve_push(moment_ctx_t ctx, const uint64_t* inbox, const int64_t* inbox_count,
                                                 int64_t cap, void* const* peer_out, void* stream) {
    MOMENT_TRY(check_ctx(ctx, "moment_relay_serve_push"));
    if (cap < 0 || !inbox || !inbox_count || !peer_out) return fail(MOMENT_EINVAL, "moment_relay_serve_push: null argument");
    if (ctx->n_bins <= 0) return fail(MOMENT_EINVAL, "moment_relay_serve_push: ctx has no bins");
    if (cap * (ctx->row_bytes / 16) >= (int64_t(1) << 40))
        return fail(MOMENT_EUNSUPPORTED, "moment_relay_serve_push: cap %lld too large", (long long)cap);
    return launch_relay_serve_push(ctx, inbox, inbox_count, cap, peer_out, static_cast<cudaStream_t>(stream));
}

// ---- cross-process device memory (peer HBM bins of other ranks) -------------------------------------
static_assert(sizeof(cudaIpcMemHandle_t) == MOMENT_IPC_HANDLE_BYTES, "IPC handle size");

extern "C" moment_status moment_ipc_export(const void* dptr, uint8_t* handle, int64_t* offset) {
    if (!dptr || !handle || !offset) return fail(MOMENT_EINVAL, "moment_ipc_export: null argument");
    // the handle names the whole allocation: report dptr's offset from its base (cuMemGetAddressRange,
    // resolved from the driver at run time so the library does not link libcuda)
    using range_fn = int (*)(unsigned long long*, size_t*, unsigned long long);
    static range_fn get_range = nullptr;
    if (!get_range) {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        MOMENT_TRY(cuda_check(cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q),
                              "moment_ipc_export: driver entry point"));
        if (!fn || q != cudaDriverEntryPointSuccess) return fail(MOMENT_ECUDA, "moment_ipc_export: cuMemGetAddressRange missing");
        get_range = reinterpret_cast<range_fn>(fn);
    }
    unsigned long long base = 0;
    size_t size = 0;
    if (get_range(&base, &size, reinterpret_cast<unsigned long long>(dptr)) != 0)
        return fail(MOMENT_ECUDA, "moment_ipc_export: cuMemGetAddressRange failed");
    cudaIpcMemHandle_t h;
    MOMENT_TRY(cuda_check(cudaIpcGetMemHandle(&h, reinterpret_cast<void*>(base)), "moment_ipc_export"));
    std::memcpy(handle, &h, sizeof(h));
    *offset = (int64_t)(reinterpret_cast<unsigned long long>(dptr) - base);
    return MOMENT_OK;
}

// An allocation can be opened only once per process, but several exported buffers may live in one
// allocation (a caching allocator's segment): imports are reference-counted per handle.
namespace {
std::mutex g_ipc_mu;
struct IpcMapping {
    std::string handle;
    void* base;
    int refs;
};
std::vector<IpcMapping> g_ipc;
}  // namespace

extern "C" moment_status moment_ipc_import(const uint8_t* handle, void** dptr) {
    if (!dptr || !handle) return fail(MOMENT_EINVAL, "moment_ipc_import: null argument");
    std::lock_guard<std::mutex> lock(g_ipc_mu);
    const std::string key(reinterpret_cast<const char*>(handle), MOMENT_IPC_HANDLE_BYTES);
    for (auto& m : g_ipc)
        if (m.handle == key) {
            m.refs++;
            *dptr = m.base;
            return MOMENT_OK;
        }
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle, sizeof(h));
    MOMENT_TRY(cuda_check(cudaIpcOpenMemHandle(dptr, h, cudaIpcMemLazyEnablePeerAccess), "moment_ipc_import"));
    g_ipc.push_back({key, *dptr, 1});
    return MOMENT_OK;
}

extern "C" moment_status moment_ipc_close(void* dptr) {
    std::lock_guard<std::mutex> lock(g_ipc_mu);
    for (size_t i = 0; i < g_ipc.size(); i++)
        if (g_ipc[i].base == dptr) {
            if (--g_ipc[i].refs > 0) return MOMENT_OK;
            g_ipc.erase(g_ipc.begin() + (long)i);
            break;
        }
    return cuda_check(cudaIpcCloseMemHandle(dptr), "moment_ipc_close");
}
