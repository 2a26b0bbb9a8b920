/*
 * moment.h — C ABI of the B200-native Moment hot path (Shi et al., "Moment: Co-optimizing Physical
 * Communication Topology and Data Placement for Multi-GPU Out-of-core GNN Training", SC '25).
 *
 * Citations "P:Lnnn" are lines of the paper text (/root/reference/PAPER.md at build time; the file is
 * not needed at run time). Readings of ambiguous passages are DESIGN.md §3 items "R#".
 *
 * Conventions (all entry points):
 *  - Every call returns moment_status: MOMENT_OK (0) or a negative error code. A human-readable message
 *    for the last failing call on the calling thread is returned by moment_last_error().
 *  - Plain pointers and sizes only. "host" pointers are ordinary CPU memory; "device" pointers are CUDA
 *    device (or UVA-mapped) memory of the context's device. Streams are passed as void* (cudaStream_t;
 *    NULL = legacy default stream).
 *  - Ownership: every array passed in stays owned by the caller. Opaque handles (topo, plan, ctx) are
 *    owned by the library and released with the matching *_free call. A ctx RETAINS the device pointers
 *    given to moment_ctx_create (CSR, bins, placement map); the caller keeps them alive until ctx_free.
 *  - Units: bytes, microseconds (us), bytes/us (= MB/s); all int64. Vertex ids are int64 at the boundary.
 *  - Device calls enqueue on the stream and return; argument, shape and range errors are detected on the
 *    host before anything is enqueued (MOMENT_EINVAL / MOMENT_EOVERFLOW). Asynchronous CUDA faults surface
 *    at the next call as MOMENT_ECUDA. No device call synchronises the host or allocates memory: every
 *    workspace is sized once in moment_ctx_create, so the calls are CUDA-graph capturable.
 *  - Determinism: sample outputs are a bitwise function of (CSR, seeds, fanout, rng_seed, flags),
 *    independent of launch configuration; gathered rows are a bitwise function of (ids, feature rows),
 *    independent of placement and routing.
 */
#ifndef MOMENT_H
#define MOMENT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t moment_status;
enum {
    MOMENT_OK = 0,
    MOMENT_EINVAL = -1,       /* bad argument, shape, id or graph */
    MOMENT_ENOMEM = -2,       /* host or device allocation failed */
    MOMENT_ECUDA = -3,        /* CUDA runtime error (message holds cudaGetErrorString) */
    MOMENT_ENCCL = -4,        /* reserved: collective transport error */
    MOMENT_EINFEASIBLE = -5,  /* demand cannot be met / knapsack capacities too small */
    MOMENT_EOVERFLOW = -6,    /* a capacity or workspace bound is too small (message holds the need) */
    MOMENT_EUNSUPPORTED = -7, /* valid request outside what this build implements */
    MOMENT_ETIMEDOUT = -8     /* cross-GPU wait exceeded its watchdog */
};

/* "virtual edges have infinite bandwidth" (Figure 9 caption; c(v_c, t) = inf) */
#define MOMENT_CAP_INF INT64_MAX

const char* moment_last_error(void);
/* Library version, (major << 16) | minor. */
int32_t moment_version(void);

/* ================================================================================================
 * P1 — communication topology graph (§3.2)
 * G = (V, E), V = V_s (storage) ∪ V_c (computation) ∪ V_i (interconnect) ∪ {s, t};
 * E = E_p (physical) ∪ E_v (virtual); flow direction source -> storage -> interconnect -> computation
 * -> sink. Capacity c(u, v) = profiled throughput upper limit, int64 bytes/us.
 * ================================================================================================ */
enum { MOMENT_NODE_SOURCE = 0, MOMENT_NODE_SINK = 1, MOMENT_NODE_STORAGE = 2, MOMENT_NODE_INTERCONNECT = 3,
       MOMENT_NODE_COMPUTE = 4 };
/* Storage hierarchy GPU > CPU > SSD: tier rank = tier - 1 (smaller is better). */
enum { MOMENT_TIER_NONE = 0, MOMENT_TIER_GPU_HBM = 1, MOMENT_TIER_HOST_DRAM = 2, MOMENT_TIER_SSD = 3 };

typedef struct {
    int32_t kind;     /* MOMENT_NODE_* */
    int32_t tier;     /* MOMENT_TIER_* (STORAGE nodes); NONE otherwise */
    int32_t device;   /* GPU rank for HBM storage / COMPUTE nodes, NUMA node for host storage, else -1 */
    int32_t reserved; /* must be 0 */
} moment_node;

typedef struct {
    int32_t from, to; /* node indices */
    int64_t cap;      /* bytes/us, >= 0, or MOMENT_CAP_INF */
} moment_link;

typedef struct moment_topo_s* moment_topo_t;

/* Validate and build the graph. Allowed links: SOURCE->STORAGE, STORAGE->INTERCONNECT,
 * STORAGE->COMPUTE, INTERCONNECT->INTERCONNECT, INTERCONNECT->COMPUTE, COMPUTE->SINK. At most one
 * SOURCE and one SINK; if absent they are appended (source = n_nodes, sink = n_nodes + 1, in that order).
 * Every STORAGE node without a source link gets s->v_s with c(s, v_s) = sum of its outgoing capacities
 * ("c(s, v_s) = c(v_s, v_i)", R8), every COMPUTE node without a sink link gets v_c->t = INF
 * (P:L221). Added links are appended after the caller's links, storage nodes first, in node order.
 * nodes/links: host arrays, copied. Errors: EINVAL (kind, index, self-loop, negative capacity, direction). */
moment_status moment_topology(const moment_node* nodes, int32_t n_nodes, const moment_link* links,
                              int32_t n_links, moment_topo_t* out);
/* Sizes of the augmented graph and the indices of s and t. Any out pointer may be NULL. */
moment_status moment_topology_info(moment_topo_t topo, int32_t* n_nodes, int32_t* n_links, int32_t* source,
                                   int32_t* sink);
/* Copy the augmented graph into caller arrays of the sizes reported by moment_topology_info. */
moment_status moment_topology_export(moment_topo_t topo, moment_node* nodes, moment_link* links);
moment_status moment_topology_free(moment_topo_t topo);

/* ================================================================================================
 * P3 — rate max-flow (§3.2 LP): maximise F = net flow out of s subject to 0 <= f <= c
 * and conservation at every node other than s, t (R7, R9 garbles). Dinic's algorithm.
 * value: F (bytes/us). link_flow: host int64[n_links] (augmented graph) or NULL. Max-flow values are
 * unique; per-link flows are not (R20) — callers check them by certificate.
 * Errors: EINVAL if an s-t path of INF links exists (unbounded), EOVERFLOW if F exceeds int64.
 * ================================================================================================ */
moment_status moment_maxflow(moment_topo_t topo, int64_t* value, int64_t* link_flow);

/* ================================================================================================
 * P4 — DDAK placement (§3.3, Eq. 2 at P:L247; readings R13-R17)
 * Vertices sorted by (hotness desc, id asc); for each pool of `pool` vertices the bin with the least
 * Eq. 2 priority (A/T)(U/C) among the non-full bins of the best tier that has traffic takes as many as fit.
 * ================================================================================================ */
enum { MOMENT_PLACE_DDAK = 0, MOMENT_PLACE_HASH = 1 };

typedef struct {
    int64_t n_vertices;
    const uint64_t* hotness;          /* host [n_vertices]: pre-sampling access counts */
    int32_t n_bins;                   /* storage bins */
    const int32_t* bin_node;          /* host [n_bins]: topology STORAGE node of each bin, or NULL = the
                                         topology's STORAGE nodes in node order (topo required) */
    const int32_t* bin_tier;          /* host [n_bins]: MOMENT_TIER_*, or NULL = from the topology */
    const int64_t* bin_capacity_rows; /* host [n_bins]: Bin_Capacity in rows (R6) */
    const int64_t* bin_traffic;       /* host [n_bins]: Bin_traffic, or NULL = f(s, bin) of the rate
                                         max-flow of topo ("modeled by maximum flow", R7) */
    int64_t pool;                     /* vertices per decision; <= 0 means 100 */
    int32_t mode;                     /* MOMENT_PLACE_DDAK, or MOMENT_PLACE_HASH (uniform baseline) */
    int64_t replicate_rows;           /* r >= 0 (DDAK mode only; R25): the r first vertices
                                         of the DDAK order are copied into EVERY GPU_HBM bin at slots 0..r-1
                                         (bin_of = MOMENT_BIN_REPLICA, slot_of = position in the order); the
                                         other vertices are placed by DDAK over the GPU bins' capacities minus
                                         r (their slots start at r) and the other bins unchanged. Requires
                                         r <= every GPU bin's capacity. 0 = plain DDAK (bit-identical). */
    int32_t traffic_mode;             /* when bin_traffic is NULL: MOMENT_TRAFFIC_RATE_FLOW (0) = f(s, b) of
                                         one rate max-flow (non-unique, R7: a symmetric box can give
                                         one of two equal host bins all the flow and the other none), or
                                         MOMENT_TRAFFIC_STANDALONE (1) = the max-flow from b alone to t with
                                         every other supply link cut (unique, R7's canonical mode) */
} moment_place_args;

enum { MOMENT_TRAFFIC_RATE_FLOW = 0, MOMENT_TRAFFIC_STANDALONE = 1 };

/* bin_of value of a vertex replicated in every GPU_HBM bin (replicate_rows > 0). */
#define MOMENT_BIN_REPLICA (-2)

typedef struct {
    int32_t* bin_of;           /* host [n_vertices] */
    int64_t* slot_of;          /* host [n_vertices]: row slot inside the bin, dense from 0 */
    uint64_t* bin_access;      /* host [n_bins] or NULL: final Bin_access (sum of hotness) */
    int64_t* bin_rows_used;    /* host [n_bins] or NULL: final Bin_currentCapacity */
    int64_t* bin_traffic_used; /* host [n_bins] or NULL: the Bin_traffic the decision used */
    uint64_t* replica_access;  /* host [1] or NULL: sum of the hotness of the replicated vertices */
} moment_place_out;

/* topo may be NULL when bin_tier and bin_traffic are given. Errors: EINVAL, EINFEASIBLE (sum of
 * capacities < n_vertices), ENOMEM. Host-only; multithreaded sort, deterministic result. */
moment_status moment_place(moment_topo_t topo, const moment_place_args* args, moment_place_out* out);
/* packed[v] = ((uint64)bin_of[v] << 40) | slot_of[v] — the device placement map layout (D3). */
moment_status moment_place_pack(int64_t n_vertices, const int32_t* bin_of, const int64_t* slot_of,
                                uint64_t* packed);
/* The device map of ONE rank when replicas exist: a MOMENT_BIN_REPLICA vertex maps to
 * (replica_bin << 40) | slot — replica_bin = that rank's own GPU_HBM bin, so every rank reads its
 * replicas locally; other vertices as moment_place_pack. Errors: EINVAL (replica_bin out of range). */
moment_status moment_place_pack_rank(int64_t n_vertices, const int32_t* bin_of, const int64_t* slot_of,
                                     int32_t replica_bin, uint64_t* packed);

/* ================================================================================================
 * P5 — time-bisection plan + quotas (ingest model R10-R12)
 * Ingest graph: the topology with supply links s->HOST bin j of k*d_j bytes (every active GPU reads d_j
 * bytes of bin j per batch), no supply on HBM bins, physical links carrying cap*T bytes in T us, v_c->t
 * INF for active GPUs only. T_ingest = min{T : maxflow(T) = sum supplies}. x[j][h] = bytes of host bin
 * j entering GPU h (path decomposition of the flow at T_ingest). GPU g then forwards x[j][h]/W_j of its
 * bin-j requests through GPU h over NVLink ("alternative paths"). T_nvlink and T_hbm are the
 * closed forms of R11; T* = max(T_ingest, T_nvlink, T_hbm).
 * ================================================================================================ */
typedef struct moment_plan_s* moment_plan_t;

typedef struct {
    int32_t k;                       /* active GPUs */
    const int32_t* gpu_node;         /* host [k]: COMPUTE node of rank r */
    const int64_t* bin_demand_bytes; /* host [n_nodes of the augmented topo]: d_b for STORAGE nodes
                                        (bytes one GPU reads from b per batch); other entries ignored */
    int64_t nvlink_cap;              /* bytes/us per GPU per direction; 0 = no NVLink (no relay) */
    int64_t hbm_cap;                 /* bytes/us per GPU, read + write */
    int64_t replica_demand_bytes;    /* bytes one GPU reads per batch from rows replicated in every active
                                        GPU's HBM (R25): a local read plus the write of the same bytes into
                                        its batch, so it adds 2x to T_hbm and nothing to NVLink or ingest */
} moment_plan_args;

moment_status moment_plan(moment_topo_t topo, const moment_plan_args* args, moment_plan_t* out);
/* Any out pointer may be NULL. link_flow: [n_links] ingest flow at T_ingest; quota: [n_nodes][k]
 * row-major x[node][rank] in bytes (non-zero only on HOST storage rows). */
moment_status moment_plan_info(moment_plan_t plan, int64_t* t_star, int64_t* t_ingest, int64_t* t_nvlink,
                               int64_t* t_hbm, int64_t* link_flow, int64_t* quota);
moment_status moment_plan_free(moment_plan_t plan);

/* ================================================================================================
 * Replication search (R25): the plan's predicted per-batch time T* as a function
 * of how many hot rows are replicated in every GPU's HBM — the paper evaluates candidate layouts by the
 * time-bisection model instead of by running them. For each candidate r:
 *   moment_place(topo, place with replicate_rows = r)                                   (P4 + R25)
 *   d_b = floor(R * A'_b / demand_batches) for every bin b (its topology node), replica demand
 *   d_rep = floor(R * A'_rep / demand_batches)   (A' = demand_counts summed over the bin's vertices: counts
 *                                                 of appearances in F_H over demand_batches batches summed
 *                                                 over all ranks; NULL = the placement's own hotness over
 *                                                 hot_batches, an in-sample estimate that over-states the
 *                                                 hit rate of the hot bins — pass held-out batches' counts)
 *   T*(r) = moment_plan(topo, k, gpu_node, d, nvlink_cap, hbm_cap, d_rep).t_star         (P5 + R25)
 * t_star[i] = T*(candidates[i]), or -1 if candidate i is infeasible (r above a GPU bin's capacity or
 * n_vertices, the rest not fitting, or the plan having no finite time). Errors: EINVAL (null or negative
 * arguments, mode not DDAK, a bin that is not a storage node). *best = the first index with the least T*, or -1 if none is feasible.
 * ================================================================================================ */
typedef struct {
    const moment_place_args* place;  /* mode must be DDAK; its replicate_rows is ignored; bin_node or the
                                        topology maps bins to storage nodes */
    int32_t k;                       /* as moment_plan_args */
    const int32_t* gpu_node;
    int64_t nvlink_cap, hbm_cap;
    int64_t row_bytes;               /* R */
    int64_t hot_batches;             /* > 0: batches place->hotness was counted over */
    const uint64_t* demand_counts;   /* host [n_vertices] or NULL (= place->hotness, hot_batches) */
    int64_t demand_batches;          /* > 0 when demand_counts is given */
    int32_t n_candidates;
    const int64_t* candidates;       /* host [n_candidates]: replicate_rows values */
} moment_replicate_args;

moment_status moment_replicate_search(moment_topo_t topo, const moment_replicate_args* args, int64_t* t_star,
                                      int32_t* best);

/* ================================================================================================
 * Device context: one per GPU rank; owns all device workspaces (no allocation on the hot path).
 * ================================================================================================ */
typedef struct moment_ctx_s* moment_ctx_t;

#define MOMENT_MAX_BINS 64

typedef struct {
    int32_t rank, world;      /* this rank, number of ranks (world = 1 for a single GPU) */
    int32_t device;           /* CUDA device ordinal of this rank */
    int64_t n_vertices;       /* |V| of the CSR graph (< 2^31) */
    int64_t max_seeds;        /* largest batch passed to moment_sample */
    int32_t max_hops;         /* largest number of hops */
    const int32_t* max_fanout;/* host [max_hops]: largest fanout per hop (workspace bounds) */
    int64_t row_bytes;        /* R: feature row bytes, multiple of 16 */
    int64_t row_stride;       /* bytes between consecutive slots of a bin (>= R, multiple of 16) */
    int32_t n_bins;           /* storage bins (<= MOMENT_MAX_BINS); 0 = no gather */
    const int32_t* bin_owner; /* host [n_bins]: owning rank of an HBM bin, -1 for a host-DRAM bin */
    void* const* bin_ptr;     /* host [n_bins]: base of each bin as addressable from THIS device: local
                                 HBM, a peer-mapped HBM pointer (NVLink) or a mapped pinned-host pointer */
    const uint64_t* placement;/* device [n_vertices]: (bin << 40) | slot (moment_place_pack), or NULL:
                                 replicated table in bin 0 at slot = vertex id (all features local) */
    const int64_t* quota;     /* host [n_bins][world] x[j][h] bytes from moment_plan_info, or NULL
                                 (every host row read directly) */
} moment_ctx_args;

moment_status moment_ctx_create(const moment_ctx_args* args, moment_ctx_t* out);
moment_status moment_ctx_free(moment_ctx_t ctx);
/* Bytes of device workspace the ctx holds. */
moment_status moment_ctx_workspace_bytes(moment_ctx_t ctx, int64_t* bytes);

/* ================================================================================================
 * H1-H3 — multi-hop neighbour sampling with dedup/relabel (R3-R6)
 * F_0 = seeds; for h < H: every v in F_h draws min(deg, fanout[h]) distinct CSR positions (Floyd with
 * Philox draws keyed on (rng_seed, v, h, i)), grouped by destination, CSR-position order;
 * F_{h+1} = F_h ++ ascending new ids; src = index of the neighbour in F_{h+1}.
 * ================================================================================================ */
typedef struct {
    const int64_t* indptr;  /* device [n_vertices + 1] */
    const int32_t* indices; /* device [n_edges] */
    int64_t n_vertices;
    int64_t n_edges;        /* = indptr[n_vertices] (the caller's contract; 0 <= n_edges < 2^40 checked) */
} moment_csr;

#define MOMENT_SAMPLE_REPLACE 1u  /* sample with replacement (k draws whenever deg > 0) */
#define MOMENT_SAMPLE_CHECK 2u    /* device-side check of seed range / uniqueness (sets EINVAL flag) */

typedef struct {
    int32_t n_hops;         /* H <= max_hops */
    const int32_t* fanout;  /* host [H], 1 <= fanout[h] <= max_fanout[h] and <= 1024 */
    uint64_t rng_seed;      /* per-batch Philox key (R1) */
    uint32_t flags;         /* MOMENT_SAMPLE_* */
} moment_sample_params;

typedef struct {
    int64_t* nodes;   /* device [cap_nodes]: F_H (F_h is a prefix of it) */
    int64_t* offsets; /* device [cap_offsets]: per hop h, |F_h|+1 offsets relative to the hop, blocks packed
                         back to back by actual size */
    int32_t* src;     /* device [cap_edges]: per hop, E_h local ids, packed back to back */
    int64_t* counts;  /* device [2H+1]: |F_0| .. |F_H|, E_0 .. E_{H-1} */
    int64_t cap_nodes, cap_offsets, cap_edges;
} moment_sample_out;

/* Upper bounds without dedup: |F_{h+1}| <= min(|F_h|(1 + f_h), n_vertices). */
moment_status moment_sample_bounds(int64_t n_seeds, const int32_t* fanout, int32_t n_hops, int64_t n_vertices,
                                   int64_t* max_nodes, int64_t* max_offsets, int64_t* max_edges);
/* seeds: device [n_seeds], distinct ids in [0, n_vertices) (checked only with MOMENT_SAMPLE_CHECK). */
moment_status moment_sample(moment_ctx_t ctx, const moment_csr* csr, const int64_t* seeds, int64_t n_seeds,
                            const moment_sample_params* params, const moment_sample_out* out, void* stream);
/* Host-side read of the device error flag raised by MOMENT_SAMPLE_CHECK (synchronises the stream). */
moment_status moment_sample_check(moment_ctx_t ctx, void* stream);

/* ================================================================================================
 * P2 — hotness by pre-sampling: hot[v] += 1 for every v in ids[0 .. *n).
 * ================================================================================================ */
moment_status moment_hotness(moment_ctx_t ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                             uint64_t* hot, void* stream);

/* ================================================================================================
 * H4 — placement lookup + bucketing ("retrieves the SSD ID and vertex offset"; R12)
 * For request i of this rank: (b, slot) = placement[ids[i]]; via = owner for HBM bins; for host bin j,
 * with n_j requests of bin j and r the rank of i among them (F_H order), slot' = floor(r W_j / n_j),
 * via = first h with slot' < cumsum_h x[j][h] (direct when W_j = 0). Queue q = b * world + via.
 * route: device int32 [max_n] (q per request); qoff: device int64 [n_bins*world + 1];
 * qpos: device int64 [max_n] (requests stably sorted by q). n_dev: device count (or NULL = max_n).
 * ================================================================================================ */
moment_status moment_bucket(moment_ctx_t ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                            int32_t* route, int64_t* qoff, int64_t* qpos, void* stream);

/* ================================================================================================
 * H5-H7 — topology-aware gather (P:L93 feature extraction; P:L391-393 relay)
 * out[i * R .. (i+1) * R) = row of ids[i], read from wherever the placement put it: local HBM, a peer's
 * HBM (NVLink load through bin_ptr) or pinned host DRAM (zero-copy PCIe read), 128-bit vectors.
 * Rows routed through a relay GPU h != rank are read by h from host DRAM and stored into this rank's out
 * over NVLink; moment_gather is then collective: one process per GPU after moment_ctx_set_exchange (one
 * enqueue per batch, below), or all ranks from one thread with moment_gather_group.
 * ids: device [max_n]; n_dev: device count or NULL (= max_n); out: device [max_n * R].
 * ================================================================================================ */
moment_status moment_gather(moment_ctx_t ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                            void* out, void* stream);

/* Collective gather of `world` ranks driven from ONE host thread on ONE stream ("logical ranks": all
 * ranks' bins and outputs addressable from the stream's device, e.g. k ranks sharing one GPU, or k
 * GPUs of one process with peer access enabled). Phase 1: bucketing + request publication for every
 * rank; phase 2: every rank's direct gather and relay service; stream order is the barrier.
 * ctxs/ids/n_dev/out: host arrays [world] of per-rank handles / device pointers. */
moment_status moment_gather_group(moment_ctx_t const* ctxs, int32_t world, const int64_t* const* ids,
                                  const int64_t* const* n_dev, int64_t max_n, void* const* out, void* stream);

/* ================================================================================================
 * H5 exchange for one process per GPU (the all-to-all transport; P:L391-393 relay through a peer).
 * Per batch, after moment_bucket (route / qoff / qpos of this rank):
 *   moment_gather_routed  : every row this rank reads itself (local HBM, peer HBM, host bins routed to
 *                           itself); rows routed through another rank are left untouched.
 *   moment_relay_pack     : words[2e] = placement word, words[2e+1] = output position of each request routed
 *                           through another rank, ordered by destination rank then bin (device int64
 *                           send_counts[world]); words: device uint64 [2 * max_n].
 *   (caller) all-to-all of the counts, then of the words (2 per request)
 *   moment_relay_serve    : rows[e] = row named by received placement word e, read by THIS rank from its own
 *                           mapping of the host bin (its PCIe link); rows: device [n][R]
 *   (caller) all-to-all of the rows back to the requesters (same splits as the words, in rows)
 *   moment_relay_scatter  : out[words[2e+1]] = rows[e] on the requester.
 * n_dev: device count or NULL (= max_n). Byte-exact with moment_gather of the same ids.
 * ================================================================================================ */
moment_status moment_gather_routed(moment_ctx_t ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                                   const int32_t* route, void* out, void* stream);
moment_status moment_relay_pack(moment_ctx_t ctx, const int64_t* ids, int64_t max_n, const int64_t* qoff,
                                const int64_t* qpos, uint64_t* words, int64_t* send_counts, void* stream);
moment_status moment_relay_serve(moment_ctx_t ctx, const uint64_t* words, const int64_t* n_dev, int64_t max_n,
                                 void* rows, void* stream);
moment_status moment_relay_scatter(moment_ctx_t ctx, const uint64_t* words, const int64_t* n_dev, int64_t max_n,
                                   const void* rows, void* out, void* stream);

/* ================================================================================================
 * H5 exchange over peer memory (one process per GPU, no all-to-all). Every rank owns an
 * inbox (device uint64 [world][cap][2]) and inbox counts (device int64 [world]); peers map them, and each
 * other's batch outputs, with moment_ipc_import (NVLink peer pointers on one node). Per batch:
 *   moment_bucket, moment_gather_routed (as above), then
 *   moment_relay_push       : the requests this rank routes through rank h are written straight into h's
 *                             inbox slot for this rank (peer stores): peer_inbox[h] = &inbox_h[self][0][0],
 *                             and their number into peer_count[h] = &count_h[self] (0 when none); entries
 *                             for h == self are ignored (may be NULL). Requests beyond cap: MOMENT_EOVERFLOW
 *                             is not detectable on the device, so the caller sizes cap >= max_n.
 *   (caller) barrier: every rank's pushes are complete and visible (moment_signal_barrier, or stream
 *                         synchronize + process barrier)
 *   moment_relay_serve_push : for every source g != self, the min(count[g], cap) requests of inbox[g] are
 *                             read from THIS rank's mapping of the host bins (its PCIe link) and stored
 *                             straight into g's output (peer stores): peer_out[g] = g's out base,
 *                             out_g[position] = row. peer_out[self] is ignored.
 *   (caller) barrier: every served row is complete before the requesters read their outputs.
 * Host arrays peer_inbox / peer_count / peer_out have `world` entries; world <= MOMENT_MAX_WORLD.
 * Byte-exact with moment_gather of the same ids.
 * ================================================================================================ */
#define MOMENT_MAX_WORLD 64

/* Device-side barrier between the two phases (and after the second), replacing "stream synchronize +
 * process barrier" (a signal barrier over symmetric memory). Every rank owns flags[world]
 * (uint64, zero-initialised, exported with moment_ipc_export); peer_flags[h] = &flags_h[self] as mapped here
 * (NULL for h == self). The kernel issues a system-scope fence, stores `epoch` (release, system scope) into
 * every peer's slot, then waits (acquire) until flags[h] >= epoch for every h != self. `epoch` must grow from
 * call to call (e.g. 1, 2, 3, ... per barrier). After timeout_ns it stops waiting and writes MOMENT_ETIMEDOUT
 * into *status_dev (device int32, may be NULL); the caller checks it when it next synchronises. Enqueued on
 * `stream`; no host synchronisation. world == 1: no-op. Errors: EINVAL. */
moment_status moment_signal_barrier(int32_t world, int32_t rank, uint64_t* const* peer_flags, const uint64_t* flags,
                                    uint64_t epoch, int64_t timeout_ns, int32_t* status_dev, void* stream);
moment_status moment_relay_push(moment_ctx_t ctx, const int64_t* ids, int64_t max_n, const int64_t* qoff,
                                const int64_t* qpos, uint64_t* const* peer_inbox, int64_t* const* peer_count,
                                void* stream);
moment_status moment_relay_serve_push(moment_ctx_t ctx, const uint64_t* inbox, const int64_t* inbox_count,
                                      int64_t cap, void* const* peer_out, void* stream);

/* ================================================================================================
 * One-call collective exchange (the ctx holds the inbox / signal pointers; P:L391-393 relay
 * through a peer). After moment_ctx_set_exchange, moment_gather and moment_step on a ctx whose quota
 * routes host rows through other ranks run the whole per-batch exchange as ONE enqueue on the stream,
 * with no host synchronisation:
 *   moment_bucket -> moment_gather_routed (this rank's own reads) -> moment_relay_push (requests stored
 *   into the relay ranks' inboxes) -> signal barrier -> moment_relay_serve_push (rows stored into the
 *   requesters' outputs) -> signal barrier.
 * The barrier epoch lives in device memory (a counter in the ctx, advanced by each barrier kernel), so the
 * sequence replays from moment_step's cached CUDA graph. Collective: every rank of the ctxs' world calls
 * moment_gather / moment_step the same number of times in the same order (a rank with nothing to gather
 * still calls, with max_n or *n_dev = 0). Peers store relayed rows into this rank's REGISTERED output,
 * so moment_gather's `out` / moment_step's `d_rows` must be args->out, and max_n <= args->cap.
 * args (device pointers, retained by the ctx until moment_ctx_free; peer pointers mapped in THIS
 * process, e.g. by moment_ipc_import; entries [rank] are ignored):
 *   cap            requests per source rank one inbox slot holds = rows of out (>= every rank's largest batch)
 *   inbox          this rank's inbox, uint64 [world][cap][2];  inbox_count: int64 [world]
 *   flags          this rank's barrier flag words, uint64 [world], zero before the first collective call
 *   out            this rank's batch output, [cap][row_bytes] bytes, 16-byte aligned
 *   peer_inbox[h]  = &inbox_h[rank][0][0];  peer_count[h] = &count_h[rank];  peer_out[h] = out_h;
 *   peer_flag[h]   = &flags_h[rank]
 *   timeout_ns     barrier watchdog (> 0): on expiry the wait ends and moment_exchange_status reports it.
 * Errors: EINVAL (null / misaligned pointer, cap < 0, timeout <= 0), EUNSUPPORTED (world > MOMENT_MAX_WORLD).
 * moment_exchange_status synchronises `stream`, then returns MOMENT_ETIMEDOUT (and clears it) if a barrier
 * of this ctx expired since the last call, else MOMENT_OK.
 * ================================================================================================ */
typedef struct {
    int64_t cap;
    uint64_t* inbox;
    int64_t* inbox_count;
    uint64_t* flags;
    void* out;
    uint64_t* peer_inbox[MOMENT_MAX_WORLD];
    int64_t* peer_count[MOMENT_MAX_WORLD];
    void* peer_out[MOMENT_MAX_WORLD];
    uint64_t* peer_flag[MOMENT_MAX_WORLD];
    int64_t timeout_ns;
} moment_exchange_args;

moment_status moment_ctx_set_exchange(moment_ctx_t ctx, const moment_exchange_args* args);
moment_status moment_exchange_status(moment_ctx_t ctx, void* stream);

/* Cross-process device memory (another rank's HBM bin mapped into this process: the NVLink peer
 * pointer of bin_ptr). export: 64-byte handle of the allocation containing dptr and dptr's byte offset in
 * it; import: map the allocation (peer access enabled lazily) and return its base (add the offset);
 * close: unmap (pass the base). Imports are reference-counted per handle (several exported buffers may share
 * one allocation): every import needs its own close, the mapping goes away with the last. */
#define MOMENT_IPC_HANDLE_BYTES 64
moment_status moment_ipc_export(const void* dptr, uint8_t* handle, int64_t* offset);
moment_status moment_ipc_import(const uint8_t* handle, void** dptr);
moment_status moment_ipc_close(void* dptr);

/* ================================================================================================
 * One whole hot-path step on device buffers: moment_sample of `seeds` followed by moment_gather of F_H
 * into d_rows (NULL: sample only; rows relayed through other ranks need moment_ctx_set_exchange, and
 * d_rows must then be its registered output: the step is then collective, see above). The 2H + 3
 * kernels are replayed from a CUDA graph cached in the ctx (captured on the first call of a given shape:
 * csr, n_seeds, fanout, flags, out and d_rows pointers; re-captured when any of them changes), so the host
 * cost per step is one graph launch. The per-batch rng_seed and seeds pointer reach the kernels through a
 * 24-byte device call block written by the graph's first node, a one-warp kernel whose parameters are
 * replaced per launch. If `stream` is being captured by the caller, the kernels are launched directly
 * instead (capture-safe). Same outputs as moment_sample + moment_gather.
 * ================================================================================================ */
moment_status moment_step(moment_ctx_t ctx, const moment_csr* csr, const int64_t* seeds, int64_t n_seeds,
                          const moment_sample_params* params, const moment_sample_out* out, void* d_rows,
                          void* stream);

/* ================================================================================================
 * End-to-end step with HOST buffers (the e2e leg of the benchmark): moves the seeds host->device, samples,
 * gathers F_H into d_rows (NULL: sample only), moves the 2H+1 counts device->host into counts_host. All of
 * it is enqueued on `stream`; counts_host is valid once the stream has completed the step (synchronise the
 * stream or an event). Pinned (page-locked, device-mapped) buffers cross PCIe inside the step's kernels: the
 * first hop reads the seeds from host memory, the compaction's last block stores the counts (no copy-engine
 * operation); pageable buffers go through cudaMemcpyAsync. seeds_host must stay unchanged until the step's
 * first kernel has run. Several steps may be in flight on different ctxs / streams.
 * ================================================================================================ */
moment_status moment_step_host(moment_ctx_t ctx, const moment_csr* csr, const int64_t* seeds_host,
                               int64_t n_seeds, const moment_sample_params* params,
                               const moment_sample_out* out, void* d_rows, int64_t* counts_host, void* stream);

/* ================================================================================================
 * Several steps in one call: the batches in flight of a pipelined loop, one per ctx. Step i is
 * moment_step(ctxs[i], csr, seeds[i], n_seeds, params with rng_seed = rng_seeds[i], &outs[i], d_rows[i],
 * streams[i]), or with counts_host != NULL moment_step_host(..., seeds[i] on the host, ..., counts_host[i],
 * streams[i]). The n ctxs must be distinct (each owns its workspace and graph); params->rng_seed is
 * ignored. Arrays are host arrays of n entries owned by the caller. Steps are validated and enqueued in
 * order; the first failing step's status is returned and the steps before it stay enqueued.
 * ================================================================================================ */
moment_status moment_step_batch(int32_t n, const moment_ctx_t* ctxs, const moment_csr* csr,
                                const int64_t* const* seeds, int64_t n_seeds, const moment_sample_params* params,
                                const uint64_t* rng_seeds, const moment_sample_out* outs, void* const* d_rows,
                                int64_t* const* counts_host, void* const* streams);

/* ================================================================================================
 * Consumer: GraphSAGE mean aggregation over one sampled block — the sparse part of a
 * layer of the model the paper trains (Eq. 1; GraphSAGE, hidden 256). The weight GEMMs,
 * activation and loss are the caller's (plain library GEMMs).
 *   out[i, :] = (1 / deg_i) * sum_{e = offsets[i]}^{offsets[i+1]-1} x[src[e], :]      (deg_i = 0 -> 0)
 * x: device [n_src][ld_x] of `dtype` (row = dim elements, dim * size a multiple of 16 bytes, <= 2048 bytes,
 * 16-byte aligned); offsets: device int64 [n_dst + 1] relative to the block (moment_sample's per-hop
 * offsets); src: device int32 [offsets[n_dst]] (< n_src, not checked); out: device [n_dst][ld_out] of
 * `dtype`. Accumulates in fp32. Enqueued on `stream`. Errors: EINVAL (shape, dtype, alignment),
 * EUNSUPPORTED (rows above 2048 bytes).
 * Backward: grad_x[src[e], :] += grad_out[i, :] / deg_i (fp32 atomics; grad_x is caller-zeroed fp32
 * [n_src][ld_gx]); the order of the additions is not fixed, so results agree to rounding, not bitwise.
 * ================================================================================================ */
enum { MOMENT_DTYPE_F32 = 0, MOMENT_DTYPE_BF16 = 1 };

moment_status moment_sage_mean(const void* x, int64_t ld_x, int32_t dtype, int64_t dim, const int64_t* offsets,
                               const int32_t* src, int64_t n_dst, void* out, int64_t ld_out, void* stream);
moment_status moment_sage_mean_backward(const void* grad_out, int64_t ld_g, int32_t dtype, int64_t dim,
                                        const int64_t* offsets, const int32_t* src, int64_t n_dst, float* grad_x,
                                        int64_t ld_gx, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* MOMENT_H */
