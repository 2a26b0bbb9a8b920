/*
 * moment_oracle.c — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded CPU oracle for the Moment (Shi et al., SC '25) hot path.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library. The product (paper_conf_sc_shi0s0x0w25_b200/) never includes, links or calls it,
 * and this file includes nothing from the product (no shared headers, helpers or constants).
 *
 * Citations: "P:Lnnn" = /root/reference/PAPER.md line nnn (section / equation named alongside).
 * Readings of ambiguous passages are the numbered items of DESIGN.md §3 ("R#").
 *
 * Contents (each function cites the passage it follows):
 *   orc_philox4x32_10 ........ counter-based RNG (Salmon et al. Philox4x32-10; R1)
 *   orc_draw / orc_uniform ... the sampler's random stream keyed on (rng_seed, node, hop, draw) (R1, R2)
 *   orc_sample_node .......... neighbour choice for one node: Floyd without replacement / with replacement (R3)
 *   orc_sample ............... multi-hop sampling + dedup/relabel ("organized into a subgraph") (R4-R6)
 *   orc_gather ............... feature extraction: out[i] = table[ids[i]]
 *   orc_maxflow .............. Edmonds-Karp on the capacity graph (§3.2 LP) (R7-R9)
 *   orc_time_bisect .......... minimum integer time T* meeting the sinks' demand (R10)
 *   orc_plan_closed_forms .... NVLink / HBM closed-form times of the ingest plan (R11)
 *   orc_quota ................ ingest quotas x[j][h]: path decomposition of a given ingest flow (R11)
 *   orc_bucket ............... per-request routing by placement + quota (R12)
 *   orc_hash_place ........... the hash-partitioning baseline placement (R24)
 *   orc_ddak ................. data-distribution-aware knapsack, Eq. 2 (R13-R17)
 *   orc_ddak_replicate ....... the same with the r hottest rows replicated in every GPU bin (R25)
 *   orc_sage_mean(_backward) . GraphSAGE mean aggregation over a sampled block and its adjoint (Eq. 1)
 *
 * Parity status of every function is listed in DESIGN.md §4 with its pins (tests/test_oracle_*.py).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORC_OK 0
#define ORC_EINVAL (-1)
#define ORC_ENOMEM (-2)
#define ORC_EINFEASIBLE (-5)
#define ORC_EOVERFLOW (-6)
#define ORC_INF INT64_MAX

/* ------------------------------------------------------------------------------------------------
 * Philox4x32-10 (R1). Round function: two 32x32->64 multiplies by M0, M1; key bumped by W0, W1
 * between rounds; 10 rounds. Written from the published algorithm (Salmon et al., SC '11).
 * ------------------------------------------------------------------------------------------------ */
void orc_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
    uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
    uint32_t k0 = key_in[0], k1 = key_in[1];
    for (int round = 0; round < 10; round++) {
        uint64_t p0 = (uint64_t)0xD2511F53u * (uint64_t)c0;
        uint64_t p1 = (uint64_t)0xCD9E8D57u * (uint64_t)c2;
        uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
        uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
        uint32_t n0 = hi1 ^ c1 ^ k0;
        uint32_t n1 = lo1;
        uint32_t n2 = hi0 ^ c3 ^ k1;
        uint32_t n3 = lo0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
        if (round < 9) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* draw(rng_seed, v, h, i) = word (i & 3) of Philox(ctr = {lo32 v, hi32 v, h, i >> 2},
 * key = {lo32 rng_seed, hi32 rng_seed}) (R1: keyed on (batch seed, hop, node), BASELINE north_star). */
uint32_t orc_draw(uint64_t rng_seed, int64_t v, int32_t h, int64_t i) {
    uint32_t ctr[4], key[2], out[4];
    ctr[0] = (uint32_t)((uint64_t)v & 0xFFFFFFFFu);
    ctr[1] = (uint32_t)((uint64_t)v >> 32);
    ctr[2] = (uint32_t)h;
    ctr[3] = (uint32_t)(i >> 2);
    key[0] = (uint32_t)(rng_seed & 0xFFFFFFFFu);
    key[1] = (uint32_t)(rng_seed >> 32);
    orc_philox4x32_10(ctr, key, out);
    return out[i & 3];
}

/* uniform(r, m) = floor(r * m / 2^32), an integer in [0, m) for 1 <= m <= 2^32 (R2). */
uint64_t orc_uniform(uint32_t r, uint64_t m) { return ((uint64_t)r * m) >> 32; }

static int cmp_i64(const void* a, const void* b) {
    int64_t x = *(const int64_t*)a, y = *(const int64_t*)b;
    return (x > y) - (x < y);
}

/* Floyd's algorithm F2 (R3) given its k random choices t[i] in [0, d-k+i]:
 * S = {}; for i in 0..k-1: j = d-k+i; S += {t[i]} if t[i] not in S else {j}. P = sorted(S); returns k. */
int64_t orc_floyd(int64_t d, int32_t k, const int64_t* t, int64_t* P) {
    int64_t count = 0;
    for (int64_t i = 0; i < k; i++) {
        int64_t j = d - k + i;
        int in_S = 0;
        for (int64_t q = 0; q < count; q++)
            if (P[q] == t[i]) { in_S = 1; break; }
        P[count++] = in_S ? j : t[i];
    }
    qsort(P, (size_t)count, sizeof(int64_t), cmp_i64);
    return count;
}

/* Neighbour positions chosen for node v at hop h ("iteratively selecting their neighbors using
 * strategies like random sampling", P:L273 fan-outs). R3:
 *   replace:      P = [uniform(draw(v,h,i), d) for i in 0..k-1] (draw order), empty if d == 0
 *   d <= k:       P = [0 .. d-1] (take all, no draws)
 *   otherwise:    Floyd's algorithm F2: S = {}; for i in 0..k-1: j = d-k+i; t = uniform(draw(v,h,i), j+1);
 *                 S += {t} if t not in S else {j};   P = sorted(S).
 * Returns the number of positions written to P. */
int64_t orc_sample_node(uint64_t rng_seed, int64_t v, int32_t h, int64_t d, int32_t k, int32_t replace,
                        int64_t* P) {
    if (d <= 0 || k <= 0) return 0;
    if (replace) {
        for (int64_t i = 0; i < k; i++) P[i] = (int64_t)orc_uniform(orc_draw(rng_seed, v, h, i), (uint64_t)d);
        return k;
    }
    if (d <= k) {
        for (int64_t p = 0; p < d; p++) P[p] = p;
        return d;
    }
    int64_t* t = (int64_t*)malloc(sizeof(int64_t) * (size_t)k);
    for (int64_t i = 0; i < k; i++) t[i] = (int64_t)orc_uniform(orc_draw(rng_seed, v, h, i), (uint64_t)(d - k + i + 1));
    int64_t count = orc_floyd(d, k, t, P);
    free(t);
    return count;
}

/* Multi-hop sampling with dedup/relabel (Eq. 1 at P:L89 makes every node of F_h a destination of
 * hop h, R4; fanout[0] applies to the seeds, R5; F_{h+1} = F_h ++ ascending new ids, R6).
 *
 *   F_0 = seeds
 *   for h in 0..H-1:
 *     for idx, v in enumerate(F_h): for p in positions(v, h): emit (idx, indices[indptr[v] + p])
 *     new = sorted(unique(emitted ids) \ F_h);  F_{h+1} = F_h ++ new
 *     src[e] = position of emitted id e in F_{h+1};   offsets_h[idx] = first edge of idx within hop h
 *
 * Outputs: nodes[|F_H|]; offsets = concatenation over h of (|F_h|+1) entries (relative to the hop);
 * src = concatenation over h of E_h local ids; counts[2H+1] = |F_0..F_H|, E_0..E_{H-1}.
 * Errors: EINVAL (seed out of range or repeated, bad fanout), EOVERFLOW (caps too small). */
int orc_sample(const int64_t* indptr, const int32_t* indices, int64_t n, const int64_t* seeds,
               int64_t n_seeds, const int32_t* fanout, int32_t n_hops, uint64_t rng_seed, int32_t replace,
               int64_t cap_nodes, int64_t cap_edges, int64_t* nodes, int64_t* offsets, int32_t* src,
               int64_t* counts) {
    if (n_seeds < 0 || n_hops < 0 || n <= 0) return ORC_EINVAL;
    if (n_seeds > cap_nodes) return ORC_EOVERFLOW;
    int64_t* pos = (int64_t*)malloc(sizeof(int64_t) * (size_t)n); /* vertex -> local index, -1 if absent */
    if (!pos) return ORC_ENOMEM;
    for (int64_t v = 0; v < n; v++) pos[v] = -1;
    for (int64_t i = 0; i < n_seeds; i++) {
        int64_t v = seeds[i];
        if (v < 0 || v >= n || pos[v] >= 0) { free(pos); return ORC_EINVAL; }
        pos[v] = i;
        nodes[i] = v;
    }
    int64_t F = n_seeds;          /* |F_h| */
    int64_t edge_base = 0;        /* first edge of hop h in src */
    int64_t off_base = 0;         /* first entry of hop h's offsets block */
    int status = ORC_OK;
    counts[0] = F;
    int64_t maxk = 0;
    for (int32_t h = 0; h < n_hops; h++) {
        if (fanout[h] <= 0) { free(pos); return ORC_EINVAL; }
        if (fanout[h] > maxk) maxk = fanout[h];
    }
    int64_t* P = (int64_t*)malloc(sizeof(int64_t) * (size_t)(maxk > 0 ? maxk : 1));
    int64_t* emitted = NULL;
    for (int32_t h = 0; h < n_hops && status == ORC_OK; h++) {
        int32_t k = fanout[h];
        /* emit edges, grouped by destination index, CSR-position order within a destination */
        int64_t E = 0;
        for (int64_t idx = 0; idx < F; idx++) {
            int64_t v = nodes[idx];
            int64_t lo = indptr[v], d = indptr[v + 1] - indptr[v];
            offsets[off_base + idx] = E;
            int64_t c = orc_sample_node(rng_seed, v, h, d, k, replace, P);
            if (edge_base + E + c > cap_edges) { status = ORC_EOVERFLOW; break; }
            for (int64_t q = 0; q < c; q++) src[edge_base + E + q] = indices[lo + P[q]]; /* global id for now */
            E += c;
        }
        if (status != ORC_OK) break;
        offsets[off_base + F] = E;
        /* new = sorted(unique(emitted) \ F_h) */
        emitted = (int64_t*)malloc(sizeof(int64_t) * (size_t)(E > 0 ? E : 1));
        int64_t m = 0;
        for (int64_t e = 0; e < E; e++) {
            int64_t u = src[edge_base + e];
            if (pos[u] < 0) emitted[m++] = u;
        }
        qsort(emitted, (size_t)m, sizeof(int64_t), cmp_i64);
        int64_t F_next = F;
        for (int64_t q = 0; q < m; q++) {
            if (q > 0 && emitted[q] == emitted[q - 1]) continue;
            if (F_next >= cap_nodes) { status = ORC_EOVERFLOW; break; }
            nodes[F_next] = emitted[q];
            pos[emitted[q]] = F_next;
            F_next++;
        }
        free(emitted);
        emitted = NULL;
        if (status != ORC_OK) break;
        /* relabel: src = position in F_{h+1} */
        for (int64_t e = 0; e < E; e++) src[edge_base + e] = (int32_t)pos[src[edge_base + e]];
        counts[1 + h] = F_next;
        counts[1 + n_hops + h] = E;
        edge_base += E;
        off_base += F + 1;
        F = F_next;
    }
    free(P);
    free(pos);
    return status;
}

/* Feature extraction ("collecting vertex embeddings from the sampled subgraph"):
 * out[i*R : (i+1)*R] = table[ids[i]*R : (ids[i]+1)*R], byte for byte. */
void orc_gather(const uint8_t* table, int64_t row_bytes, const int64_t* ids, int64_t n, uint8_t* out) {
    for (int64_t i = 0; i < n; i++)
        memcpy(out + i * row_bytes, table + ids[i] * row_bytes, (size_t)row_bytes);
}

/* ------------------------------------------------------------------------------------------------
 * Max-flow, Edmonds-Karp (maximise F = total flow s -> t subject to 0 <= f <= c and
 * conservation at every node other than s, t; R7 objective = net flow out of s; R8 conservation).
 * Capacities are int64 bytes per microsecond; ORC_INF (INT64_MAX) means unbounded (P:L200, P:L221
 * "virtual edges have infinite bandwidth"). R9: an s->t path made only of INF links => EINVAL.
 * Residual arcs: arc 2i = link i forward (residual c - f), arc 2i+1 = link i backward (residual f).
 * BFS visits a node's arcs in link insertion order; augment along the shortest path by its bottleneck.
 * ------------------------------------------------------------------------------------------------ */
static int64_t arc_residual(const int64_t* cap, const int64_t* flow, int64_t arc) {
    int64_t i = arc >> 1;
    if (arc & 1) return flow[i];
    if (cap[i] == ORC_INF) return ORC_INF;
    return cap[i] - flow[i];
}

int orc_maxflow(int32_t n_nodes, int32_t n_links, const int32_t* from, const int32_t* to, const int64_t* cap,
                int32_t s, int32_t t, int64_t* value, int64_t* flow_out) {
    if (n_nodes <= 0 || s < 0 || t < 0 || s >= n_nodes || t >= n_nodes || s == t) return ORC_EINVAL;
    for (int32_t i = 0; i < n_links; i++) {
        if (from[i] < 0 || from[i] >= n_nodes || to[i] < 0 || to[i] >= n_nodes || cap[i] < 0) return ORC_EINVAL;
    }
    int64_t* flow = (int64_t*)calloc((size_t)(n_links > 0 ? n_links : 1), sizeof(int64_t));
    int64_t* parc = (int64_t*)malloc(sizeof(int64_t) * (size_t)n_nodes);   /* arc used to reach node */
    int32_t* queue = (int32_t*)malloc(sizeof(int32_t) * (size_t)n_nodes);
    /* adjacency: for each node, arcs in link insertion order */
    int32_t* deg = (int32_t*)calloc((size_t)n_nodes + 1, sizeof(int32_t));
    for (int32_t i = 0; i < n_links; i++) { deg[from[i] + 1]++; deg[to[i] + 1]++; }
    for (int32_t u = 0; u < n_nodes; u++) deg[u + 1] += deg[u];
    int64_t* adj = (int64_t*)malloc(sizeof(int64_t) * (size_t)(2 * n_links + 1));
    int32_t* fill = (int32_t*)calloc((size_t)n_nodes, sizeof(int32_t));
    for (int32_t i = 0; i < n_links; i++) {
        adj[deg[from[i]] + fill[from[i]]++] = 2 * (int64_t)i;
        adj[deg[to[i]] + fill[to[i]]++] = 2 * (int64_t)i + 1;
    }
    int status = ORC_OK;
    /* R9: unbounded if s reaches t through INF links only */
    {
        char* seen = (char*)calloc((size_t)n_nodes, 1);
        int32_t qh = 0, qt = 0;
        queue[qt++] = s; seen[s] = 1;
        while (qh < qt) {
            int32_t u = queue[qh++];
            for (int32_t a = deg[u]; a < deg[u + 1]; a++) {
                int64_t arc = adj[a];
                if (arc & 1) continue;
                int32_t w = to[arc >> 1];
                if (cap[arc >> 1] == ORC_INF && !seen[w]) { seen[w] = 1; queue[qt++] = w; }
            }
        }
        if (seen[t]) status = ORC_EINVAL;
        free(seen);
    }
    int64_t total = 0;
    while (status == ORC_OK) {
        for (int32_t u = 0; u < n_nodes; u++) parc[u] = -1;
        int32_t qh = 0, qt = 0;
        queue[qt++] = s;
        parc[s] = -2;
        while (qh < qt && parc[t] == -1) {
            int32_t u = queue[qh++];
            for (int32_t a = deg[u]; a < deg[u + 1]; a++) {
                int64_t arc = adj[a];
                int32_t w = (arc & 1) ? from[arc >> 1] : to[arc >> 1];
                if (parc[w] != -1) continue;
                if (arc_residual(cap, flow, arc) <= 0) continue;
                parc[w] = arc;
                queue[qt++] = w;
            }
        }
        if (parc[t] == -1) break;
        int64_t bottleneck = ORC_INF;
        for (int32_t w = t; w != s;) {
            int64_t arc = parc[w];
            int64_t r = arc_residual(cap, flow, arc);
            if (r < bottleneck) bottleneck = r;
            w = (arc & 1) ? to[arc >> 1] : from[arc >> 1];
        }
        if (bottleneck == ORC_INF) { status = ORC_EINVAL; break; }
        for (int32_t w = t; w != s;) {
            int64_t arc = parc[w];
            if (arc & 1) flow[arc >> 1] -= bottleneck;
            else {
                if (flow[arc >> 1] > ORC_INF - 1 - bottleneck) { status = ORC_EOVERFLOW; break; }
                flow[arc >> 1] += bottleneck;
            }
            w = (arc & 1) ? to[arc >> 1] : from[arc >> 1];
        }
        if (status != ORC_OK) break;
        if (total > ORC_INF - 1 - bottleneck) { status = ORC_EOVERFLOW; break; }
        total += bottleneck;
    }
    if (status == ORC_OK) {
        *value = total;
        if (flow_out) memcpy(flow_out, flow, sizeof(int64_t) * (size_t)n_links);
    }
    free(flow); free(parc); free(queue); free(deg); free(adj); free(fill);
    return status;
}

/* ------------------------------------------------------------------------------------------------
 * Time-bisection ("a time-bisection Ford-Fulkerson method ... to estimate the minimum time
 * required to reach the sink's total access demand"). R10: supply links (is_supply[i] = 1) carry
 * bytes (the demand placed on a storage node); every other finite link carries cap * T bytes in T
 * microseconds; INF links stay INF. T* = min{T in N : maxflow(T) = sum of supplies}; maxflow(T) is
 * non-decreasing in T, so search by doubling from T = 1, then bisection. D = 0 => T* = 0.
 * Infeasible (maxflow < D even with every physical link INF) => EINFEASIBLE.
 * ------------------------------------------------------------------------------------------------ */
static int64_t scaled_cap(int64_t c, int64_t T) {
    if (c == ORC_INF) return ORC_INF;
    const int64_t LIM = (int64_t)1 << 62;      /* finite ceiling: far above any demand we accept */
    if (c != 0 && T > LIM / c) return LIM;
    return c * T;
}

static int flow_at(int32_t n_nodes, int32_t n_links, const int32_t* from, const int32_t* to, const int64_t* cap,
                   const uint8_t* is_supply, int32_t s, int32_t t, int64_t T, int64_t* value, int64_t* flow) {
    int64_t* c = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n_links > 0 ? n_links : 1));
    for (int32_t i = 0; i < n_links; i++) c[i] = is_supply[i] ? cap[i] : (T < 0 ? ORC_INF : scaled_cap(cap[i], T));
    int st = orc_maxflow(n_nodes, n_links, from, to, c, s, t, value, flow);
    free(c);
    return st;
}

int orc_time_bisect(int32_t n_nodes, int32_t n_links, const int32_t* from, const int32_t* to, const int64_t* cap,
                    const uint8_t* is_supply, int32_t s, int32_t t, int64_t* t_star, int64_t* flow_out) {
    int64_t D = 0;
    for (int32_t i = 0; i < n_links; i++) {
        if (is_supply[i]) {
            if (cap[i] == ORC_INF || cap[i] < 0) return ORC_EINVAL;
            if (D > ((int64_t)1 << 62) - cap[i]) return ORC_EOVERFLOW;
            D += cap[i];
        }
    }
    int64_t v = 0;
    if (D == 0) {
        *t_star = 0;
        return flow_at(n_nodes, n_links, from, to, cap, is_supply, s, t, 0, &v, flow_out);
    }
    int st = flow_at(n_nodes, n_links, from, to, cap, is_supply, s, t, -1, &v, NULL);
    if (st != ORC_OK) return st;
    if (v < D) return ORC_EINFEASIBLE;
    int64_t hi = 1;
    for (;;) {
        st = flow_at(n_nodes, n_links, from, to, cap, is_supply, s, t, hi, &v, NULL);
        if (st != ORC_OK) return st;
        if (v == D) break;
        if (hi > ((int64_t)1 << 61)) return ORC_EINFEASIBLE;
        hi *= 2;
    }
    int64_t lo = hi / 2; /* maxflow(lo) < D (or lo == 0) */
    while (hi - lo > 1) {
        int64_t mid = lo + (hi - lo) / 2;
        st = flow_at(n_nodes, n_links, from, to, cap, is_supply, s, t, mid, &v, NULL);
        if (st != ORC_OK) return st;
        if (v == D) hi = mid; else lo = mid;
    }
    *t_star = hi;
    return flow_at(n_nodes, n_links, from, to, cap, is_supply, s, t, hi, &v, flow_out);
}

/* ------------------------------------------------------------------------------------------------
 * Closed-form NVLink / HBM times of a plan (R11; the paper's "alternative paths" through NVLink,
 * P:L391-393). Per GPU per batch, GPU g reads d_b bytes from storage bin b.
 *   HBM bin b owned by o: read locally when o == g, else one NVLink hop o -> g.
 *   host bin j: GPU g sends the fraction x[j][h] / W_j (W_j = sum_h x[j][h]) through GPU h (h == g: direct).
 * in_g  = sum_{b HBM, o != g} d_b + sum_j ceil(d_j * (W_j - x[j][g]) / W_j)
 * out_h = sum_{b HBM owned by h} (k-1) d_b + sum_j ceil((k-1) * d_j * x[j][h] / W_j)
 * T_nvlink = ceil(max_g max(in_g, out_g) / nvlink_cap) (0 if no NVLink bytes);
 * T_hbm = ceil(max_g (k d_{HBM_g} + sum_b d_b + 2 d_rep) / hbm_cap)   (reads of g's HBM bin by all k GPUs
 *         plus the writes of g's own batch buffer; d_rep = bytes g reads from rows replicated in every
 *         GPU's HBM, read locally and written into its batch, R25). Each relay term is rounded up to
 *         whole bytes (R11).
 * Inputs are indexed by rank 0..k-1: hbm_owner[b] = owning rank, or -1 for host bins; x is [n_bins][k].
 * ------------------------------------------------------------------------------------------------ */
static int64_t ceil_div_u128(unsigned __int128 a, unsigned __int128 b) {
    return (int64_t)((a + b - 1) / b);
}

int orc_plan_closed_forms(int32_t k, int32_t n_bins, const int32_t* hbm_owner, const int64_t* d,
                          const int64_t* x, int64_t nvlink_cap, int64_t hbm_cap, int64_t replica_d,
                          int64_t* t_nvlink, int64_t* t_hbm) {
    int64_t max_link = 0, max_hbm = 0;
    /* R25: replicated rows are read from g's own HBM and written into its batch: 2 replica_d on g's
     * HBM, nothing on NVLink */
    int64_t total_d = 2 * replica_d;
    for (int32_t b = 0; b < n_bins; b++) total_d += d[b];
    for (int32_t g = 0; g < k; g++) {
        int64_t in_g = 0, out_g = 0, hbm_g = total_d;
        for (int32_t b = 0; b < n_bins; b++) {
            if (hbm_owner[b] >= 0) {
                if (hbm_owner[b] != g) in_g += d[b];
                else { out_g += (int64_t)(k - 1) * d[b]; hbm_g += (int64_t)k * d[b]; }
            } else {
                int64_t W = 0;
                for (int32_t h = 0; h < k; h++) W += x[(int64_t)b * k + h];
                if (W == 0 || d[b] == 0) continue;
                in_g += ceil_div_u128((unsigned __int128)d[b] * (unsigned __int128)(W - x[(int64_t)b * k + g]),
                                      (unsigned __int128)W);
                out_g += ceil_div_u128((unsigned __int128)(k - 1) * (unsigned __int128)d[b] *
                                           (unsigned __int128)x[(int64_t)b * k + g],
                                       (unsigned __int128)W);
            }
        }
        int64_t m = in_g > out_g ? in_g : out_g;
        if (m > max_link) max_link = m;
        if (hbm_g > max_hbm) max_hbm = hbm_g;
    }
    if (max_link > 0 && nvlink_cap <= 0) return ORC_EINFEASIBLE;
    *t_nvlink = max_link == 0 ? 0 : ceil_div_u128((unsigned __int128)max_link, (unsigned __int128)nvlink_cap);
    if (hbm_cap <= 0) return ORC_EINVAL;
    *t_hbm = ceil_div_u128((unsigned __int128)max_hbm, (unsigned __int128)hbm_cap);
    return ORC_OK;
}

/* ------------------------------------------------------------------------------------------------
 * Ingest quotas ("time-bisection Ford-Fulkerson"; the paper does not say how the single-
 * commodity flow becomes per-GPU routing, R11). x[j][h] = bytes of host bin j that enter through GPU
 * h's port = a path decomposition of the GIVEN ingest flow f (flows are not unique, so the quotas are a
 * function of the flow the planner produced). The decomposition is the textbook one (follow positive
 * flow from the source, cancel any cycle met on the way), in this fixed order:
 *   for every supply link s -> j in link order, while its remaining flow is > 0:
 *     walk from j; at node u:
 *       if u is an active GPU (rank_of_node[u] >= 0) and one of its links into t has remaining flow
 *         (the first such in link order), the walk ends there;
 *       else follow the first out-link of u in link order (not into t) with remaining flow;
 *       if that link leads back to a node w already on the walk, the closed cycle (the walk's links
 *         from w on, plus this link) loses its minimum remaining flow on every link, the walk is cut
 *         back to w, and it resumes from w;
 *     m = minimum remaining flow over the supply link and the walk's links; subtract m from each;
 *     x[j][rank of the walk's last GPU] += m.
 * x is [n_nodes][k] (rows of non-host nodes stay 0). Returns ORC_EINVAL if the flow is not
 * conserved (a walk gets stuck).
 * ------------------------------------------------------------------------------------------------ */
int orc_quota(int32_t n_nodes, int32_t n_links, const int32_t* from, const int32_t* to, const int64_t* flow,
              int32_t s, int32_t t, int32_t k, const int32_t* rank_of_node, int64_t* x) {
    if (n_nodes <= 0 || n_links < 0 || k <= 0) return ORC_EINVAL;
    int64_t* rem = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n_links > 0 ? n_links : 1));
    int32_t* walk = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n_links + 1)); /* link indices */
    int32_t* at = (int32_t*)malloc(sizeof(int32_t) * (size_t)n_nodes);         /* position on walk or -1 */
    if (!rem || !walk || !at) { free(rem); free(walk); free(at); return ORC_ENOMEM; }
    for (int32_t e = 0; e < n_links; e++) rem[e] = flow[e];
    for (int64_t i = 0; i < (int64_t)n_nodes * k; i++) x[i] = 0;
    int rc = ORC_OK;
    for (int32_t e0 = 0; e0 < n_links && rc == ORC_OK; e0++) {
        if (from[e0] != s) continue;
        int32_t j = to[e0];
        while (rem[e0] > 0) {
            int32_t len = 0;
            for (int32_t v = 0; v < n_nodes; v++) at[v] = -1;
            int32_t u = j;
            at[u] = 0;
            int32_t last_gpu = -1;
            for (;;) {
                int32_t sink = -1;
                if (rank_of_node[u] >= 0)
                    for (int32_t e = 0; e < n_links; e++)
                        if (from[e] == u && to[e] == t && rem[e] > 0) { sink = e; break; }
                if (sink >= 0) { walk[len++] = sink; last_gpu = u; break; }
                int32_t nxt = -1;
                for (int32_t e = 0; e < n_links; e++)
                    if (from[e] == u && to[e] != t && rem[e] > 0) { nxt = e; break; }
                if (nxt < 0) { rc = ORC_EINVAL; break; }
                int32_t w = to[nxt];
                if (at[w] >= 0) {
                    /* cycle: walk[at[w] .. len-1] + nxt */
                    int64_t m = rem[nxt];
                    for (int32_t q = at[w]; q < len; q++) if (rem[walk[q]] < m) m = rem[walk[q]];
                    rem[nxt] -= m;
                    for (int32_t q = at[w]; q < len; q++) rem[walk[q]] -= m;
                    for (int32_t q = at[w]; q < len; q++) at[to[walk[q]]] = -1;
                    len = at[w];
                    at[w] = len;
                    u = w;
                    continue;
                }
                walk[len++] = nxt;
                at[w] = len;
                u = w;
            }
            if (rc != ORC_OK) break;
            int64_t m = rem[e0];
            for (int32_t q = 0; q < len; q++) if (rem[walk[q]] < m) m = rem[walk[q]];
            rem[e0] -= m;
            for (int32_t q = 0; q < len; q++) rem[walk[q]] -= m;
            x[(int64_t)j * k + rank_of_node[last_gpu]] += m;
        }
    }
    free(rem); free(walk); free(at);
    return rc;
}

/* ------------------------------------------------------------------------------------------------
 * Hash-partitioning baseline placement (the systems Moment compares against partition
 * embeddings by hash; R24): vertices in id order; bin = splitmix64(v) mod n_bins (the splitmix64
 * output function of Steele et al. with state v); a full bin passes the vertex to the next bin index
 * (cyclically); slot = the bin's fill count at that moment. ORC_EINFEASIBLE if the capacities hold
 * fewer than n rows.
 * ------------------------------------------------------------------------------------------------ */
static uint64_t orc_splitmix64(uint64_t state) {
    uint64_t z = state + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

int orc_hash_place(int64_t n, int32_t n_bins, const int64_t* cap_rows, int32_t* bin_of, int64_t* slot_of,
                   int64_t* used) {
    if (n < 0 || n_bins <= 0) return ORC_EINVAL;
    int64_t total = 0;
    for (int32_t b = 0; b < n_bins; b++) { used[b] = 0; total += cap_rows[b]; }
    if (total < n) return ORC_EINFEASIBLE;
    for (int64_t v = 0; v < n; v++) {
        int32_t b = (int32_t)(orc_splitmix64((uint64_t)v) % (uint64_t)n_bins);
        while (used[b] >= cap_rows[b]) b = (b + 1) % n_bins;
        bin_of[v] = b;
        slot_of[v] = used[b];
        used[b]++;
    }
    return ORC_OK;
}

/* ------------------------------------------------------------------------------------------------
 * Request routing ("each GPU retrieves the SSD ID and vertex offset, then initiates parallel
 * IO requests"; R12 routing by quota). For rank g and request i (a position in F_H):
 *   (b, slot) = placement of ids[i]
 *   HBM bin of owner o            -> via = o        (local read if o == g, NVLink peer load otherwise)
 *   host bin j, n_j = #requests of g on bin j, r = rank of i among them in F_H order,
 *   W = sum_h x[j][h]             -> slot' = floor(r W / n_j); via = first h with slot' < cumsum_h x[j][.]
 *                                    (W == 0: via = g, direct)
 * Queue q = b * k + via. Output: route[i] = q; queues stable-sorted by (q, i): qoff[Q+1], qpos[n].
 * ------------------------------------------------------------------------------------------------ */
int orc_bucket(int32_t g, int32_t k, int32_t n_bins, const int32_t* hbm_owner, const int64_t* x,
               const int32_t* bin_of_id, int64_t n, int32_t* route, int64_t* qoff, int64_t* qpos) {
    if (k <= 0 || n_bins <= 0 || g < 0 || g >= k || n < 0) return ORC_EINVAL;
    int64_t* n_j = (int64_t*)calloc((size_t)n_bins, sizeof(int64_t));
    int64_t* r_j = (int64_t*)calloc((size_t)n_bins, sizeof(int64_t));
    for (int64_t i = 0; i < n; i++) {
        int32_t b = bin_of_id[i];
        if (b < 0 || b >= n_bins) { free(n_j); free(r_j); return ORC_EINVAL; }
        n_j[b]++;
    }
    for (int64_t i = 0; i < n; i++) {
        int32_t b = bin_of_id[i];
        int32_t via;
        if (hbm_owner[b] >= 0) {
            via = hbm_owner[b];
        } else {
            int64_t W = 0;
            for (int32_t h = 0; h < k; h++) W += x[(int64_t)b * k + h];
            int64_t r = r_j[b]++;
            if (W == 0) {
                via = g;
            } else {
                int64_t s = (int64_t)(((unsigned __int128)r * (unsigned __int128)W) / (unsigned __int128)n_j[b]);
                int64_t cum = 0;
                via = k - 1;
                for (int32_t h = 0; h < k; h++) {
                    cum += x[(int64_t)b * k + h];
                    if (s < cum) { via = h; break; }
                }
            }
        }
        route[i] = b * k + via;
    }
    int64_t Q = (int64_t)n_bins * k;
    for (int64_t q = 0; q <= Q; q++) qoff[q] = 0;
    for (int64_t i = 0; i < n; i++) qoff[route[i] + 1]++;
    for (int64_t q = 0; q < Q; q++) qoff[q + 1] += qoff[q];
    int64_t* fillq = (int64_t*)calloc((size_t)Q, sizeof(int64_t));
    for (int64_t i = 0; i < n; i++) qpos[qoff[route[i]] + fillq[route[i]]++] = i;
    free(fillq); free(n_j); free(r_j);
    return ORC_OK;
}

/* ------------------------------------------------------------------------------------------------
 * DDAK, data-distribution-aware knapsack (Eq. 2 at P:L247). R13-R17:
 *   order = vertices by (hotness desc, id asc)                                       (R17 ties)
 *   tiers by rank: GPU HBM (0) > host DRAM (1) > SSD (2)                            (R14)
 *   for each group of `pool` consecutive vertices of order (R15):
 *     while the group is not empty:
 *       cand = non-full bins of the best tier that has a non-full bin with traffic > 0;
 *              if none: all non-full bins; if none: EINFEASIBLE
 *       b* = argmin over cand of priority_b = (A_b / T_b) * (U_b / C_b)           (Eq. 2; R13 argmin)
 *            T_b = 0 => +inf; ties -> less filled (U_b / C_b), then better tier, then lower index (R16)
 *       take m = min(|group|, C_b* - U_b*) vertices in order; slot_of = U_b*, U_b*+1, ...
 *       A_b* += their hotness; U_b* += m                                            (P:L252 re-evaluate)
 * A = Bin_access (cumulative hotness), T = Bin_traffic, U = Bin_currentCapacity (rows), C = Bin_Capacity.
 * Exact comparison: A_a U_a T_b C_b < A_b U_b T_a C_a evaluated in 256-bit integers.
 * ------------------------------------------------------------------------------------------------ */
typedef struct { uint64_t w[4]; } u256;

static u256 mul128x128(unsigned __int128 a, unsigned __int128 b) {
    uint64_t al[2] = {(uint64_t)a, (uint64_t)(a >> 64)};
    uint64_t bl[2] = {(uint64_t)b, (uint64_t)(b >> 64)};
    u256 r = {{0, 0, 0, 0}};
    for (int i = 0; i < 2; i++) {
        unsigned __int128 carry = 0;
        for (int j = 0; j < 2; j++) {
            unsigned __int128 cur = (unsigned __int128)al[i] * bl[j] + r.w[i + j] + carry;
            r.w[i + j] = (uint64_t)cur;
            carry = cur >> 64;
        }
        int p = i + 2;
        while (carry) {
            unsigned __int128 cur = (unsigned __int128)r.w[p] + carry;
            r.w[p] = (uint64_t)cur;
            carry = cur >> 64;
            p++;
        }
    }
    return r;
}

static int cmp256(u256 a, u256 b) {
    for (int i = 3; i >= 0; i--) {
        if (a.w[i] < b.w[i]) return -1;
        if (a.w[i] > b.w[i]) return 1;
    }
    return 0;
}

/* -1 if priority(a) < priority(b), 0 if equal, 1 if greater. */
static int priority_cmp(uint64_t Aa, int64_t Ua, int64_t Ta, int64_t Ca, uint64_t Ab, int64_t Ub, int64_t Tb,
                        int64_t Cb) {
    int inf_a = (Ta == 0), inf_b = (Tb == 0);
    if (inf_a && inf_b) return 0;
    if (inf_a) return 1;
    if (inf_b) return -1;
    u256 lhs = mul128x128((unsigned __int128)Aa * (uint64_t)Ua, (unsigned __int128)(uint64_t)Tb * (uint64_t)Cb);
    u256 rhs = mul128x128((unsigned __int128)Ab * (uint64_t)Ub, (unsigned __int128)(uint64_t)Ta * (uint64_t)Ca);
    return cmp256(lhs, rhs);
}

static const uint64_t* g_hot_for_sort;
static int cmp_hot_desc(const void* a, const void* b) {
    int64_t x = *(const int64_t*)a, y = *(const int64_t*)b;
    uint64_t hx = g_hot_for_sort[x], hy = g_hot_for_sort[y];
    if (hx != hy) return hx > hy ? -1 : 1;
    return (x > y) - (x < y);
}

int orc_ddak(int64_t n, const uint64_t* hotness, int32_t n_bins, const int32_t* tier_rank, const int64_t* cap_rows,
             const int64_t* traffic, int64_t pool, int32_t* bin_of, int64_t* slot_of, uint64_t* access_out,
             int64_t* used_out) {
    if (n < 0 || n_bins <= 0 || pool <= 0) return ORC_EINVAL;
    for (int32_t b = 0; b < n_bins; b++)
        if (cap_rows[b] < 0 || traffic[b] < 0 || tier_rank[b] < 0) return ORC_EINVAL;
    int64_t* order = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    if (!order) return ORC_ENOMEM;
    for (int64_t v = 0; v < n; v++) order[v] = v;
    g_hot_for_sort = hotness;
    qsort(order, (size_t)n, sizeof(int64_t), cmp_hot_desc);
    uint64_t* A = (uint64_t*)calloc((size_t)n_bins, sizeof(uint64_t));
    int64_t* U = (int64_t*)calloc((size_t)n_bins, sizeof(int64_t));
    int status = ORC_OK;
    for (int64_t g0 = 0; g0 < n && status == ORC_OK; g0 += pool) {
        int64_t g1 = g0 + pool < n ? g0 + pool : n;
        int64_t next = g0;
        while (next < g1) {
            /* best tier having a non-full bin with traffic > 0 */
            int32_t best_tier = -1;
            for (int32_t b = 0; b < n_bins; b++)
                if (U[b] < cap_rows[b] && traffic[b] > 0 && (best_tier < 0 || tier_rank[b] < best_tier))
                    best_tier = tier_rank[b];
            int32_t bstar = -1;
            for (int32_t b = 0; b < n_bins; b++) {
                if (U[b] >= cap_rows[b]) continue;
                if (best_tier >= 0 && tier_rank[b] != best_tier) continue;
                if (bstar < 0) { bstar = b; continue; }
                int c = priority_cmp(A[b], U[b], traffic[b], cap_rows[b], A[bstar], U[bstar], traffic[bstar],
                                     cap_rows[bstar]);
                if (c == 0) {
                    /* R16: equal priority -> the less-filled bin, U_b / C_b < U_b* / C_b* */
                    unsigned __int128 fb = (unsigned __int128)(uint64_t)U[b] * (uint64_t)cap_rows[bstar];
                    unsigned __int128 fs = (unsigned __int128)(uint64_t)U[bstar] * (uint64_t)cap_rows[b];
                    c = fb < fs ? -1 : (fb > fs ? 1 : 0);
                }
                if (c < 0 || (c == 0 && tier_rank[b] < tier_rank[bstar])) bstar = b;
                /* equal priority, fill and tier: keep the lower index (bstar < b) */
            }
            if (bstar < 0) { status = ORC_EINFEASIBLE; break; }
            int64_t room = cap_rows[bstar] - U[bstar];
            int64_t m = g1 - next < room ? g1 - next : room;
            for (int64_t q = 0; q < m; q++) {
                int64_t v = order[next + q];
                bin_of[v] = bstar;
                slot_of[v] = U[bstar] + q;
                A[bstar] += hotness[v];
            }
            U[bstar] += m;
            next += m;
        }
    }
    if (status == ORC_OK) {
        if (access_out) memcpy(access_out, A, sizeof(uint64_t) * (size_t)n_bins);
        if (used_out) memcpy(used_out, U, sizeof(int64_t) * (size_t)n_bins);
    }
    free(order); free(A); free(U);
    return status;
}

/* ------------------------------------------------------------------------------------------------
 * Replication-aware DDAK (R25; an extension of Eq. 2):
 *   order = vertices by (hotness desc, id asc)                                            (as orc_ddak)
 *   the first r vertices of order are replicas: bin_of = -2, slot_of = position in order; each sits at
 *     that slot in EVERY GPU-tier bin (tier_rank 0), so every GPU bin needs capacity >= r
 *   the remaining vertices are placed by orc_ddak with GPU bins' capacities reduced by r; their slots in
 *     GPU bins are shifted by r (the bin holds [replicas | partition])
 * rep_access = sum of the replicas' hotness. A and U count the partition only.
 * ------------------------------------------------------------------------------------------------ */
int orc_ddak_replicate(int64_t n, const uint64_t* hotness, int32_t n_bins, const int32_t* tier_rank,
                       const int64_t* cap_rows, const int64_t* traffic, int64_t pool, int64_t r, int32_t* bin_of,
                       int64_t* slot_of, uint64_t* access_out, int64_t* used_out, uint64_t* rep_access) {
    if (n < 0 || n_bins <= 0 || pool <= 0 || r < 0 || r > n) return ORC_EINVAL;
    for (int32_t b = 0; b < n_bins; b++)
        if (tier_rank[b] == 0 && cap_rows[b] < r) return ORC_EINFEASIBLE;
    int64_t* order = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    if (!order) return ORC_ENOMEM;
    for (int64_t v = 0; v < n; v++) order[v] = v;
    g_hot_for_sort = hotness;
    qsort(order, (size_t)n, sizeof(int64_t), cmp_hot_desc);
    char* is_rep = (char*)calloc((size_t)(n > 0 ? n : 1), 1);
    uint64_t rep = 0;
    for (int64_t i = 0; i < r; i++) {
        is_rep[order[i]] = 1;
        bin_of[order[i]] = -2;
        slot_of[order[i]] = i;
        rep += hotness[order[i]];
    }
    free(order);
    /* the remaining vertices, in ascending id order (keeps orc_ddak's id tie-break) */
    int64_t m = n - r;
    int64_t* ids = (int64_t*)malloc(sizeof(int64_t) * (size_t)(m > 0 ? m : 1));
    uint64_t* sub_hot = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(m > 0 ? m : 1));
    int32_t* sub_bin = (int32_t*)malloc(sizeof(int32_t) * (size_t)(m > 0 ? m : 1));
    int64_t* sub_slot = (int64_t*)malloc(sizeof(int64_t) * (size_t)(m > 0 ? m : 1));
    int64_t* cap2 = (int64_t*)malloc(sizeof(int64_t) * (size_t)n_bins);
    int64_t j = 0;
    for (int64_t v = 0; v < n; v++)
        if (!is_rep[v]) { ids[j] = v; sub_hot[j] = hotness[v]; j++; }
    for (int32_t b = 0; b < n_bins; b++) cap2[b] = tier_rank[b] == 0 ? cap_rows[b] - r : cap_rows[b];
    int st = orc_ddak(m, sub_hot, n_bins, tier_rank, cap2, traffic, pool, sub_bin, sub_slot, access_out, used_out);
    if (st == ORC_OK) {
        for (int64_t q = 0; q < m; q++) {
            bin_of[ids[q]] = sub_bin[q];
            slot_of[ids[q]] = sub_slot[q] + (tier_rank[sub_bin[q]] == 0 ? r : 0);
        }
        if (rep_access) *rep_access = rep;
    }
    free(is_rep); free(ids); free(sub_hot); free(sub_bin); free(sub_slot); free(cap2);
    return st;
}

/* ------------------------------------------------------------------------------------------------
 * GraphSAGE mean aggregation over one sampled block (Eq. 1: the aggregate of the neighbours'
 * h_u^{l-1}; the paper's model is GraphSAGE), in fp64:
 *   out[i][c] = (1 / deg_i) * sum_{e = offsets[i]}^{offsets[i+1]-1} x[src[e]][c],  deg_i = 0 -> 0
 * and its adjoint (the backward of the same linear map):
 *   gx[src[e]][c] += g[i][c] / deg_i   for every edge e of row i
 * ------------------------------------------------------------------------------------------------ */
void orc_sage_mean(const double* x, int64_t dim, const int64_t* offsets, const int32_t* src, int64_t n_dst,
                   double* out) {
    for (int64_t i = 0; i < n_dst; i++) {
        int64_t deg = offsets[i + 1] - offsets[i];
        for (int64_t c = 0; c < dim; c++) {
            double acc = 0.0;
            for (int64_t e = offsets[i]; e < offsets[i + 1]; e++) acc += x[(int64_t)src[e] * dim + c];
            out[i * dim + c] = deg > 0 ? acc / (double)deg : 0.0;
        }
    }
}

void orc_sage_mean_backward(const double* g, int64_t dim, const int64_t* offsets, const int32_t* src, int64_t n_dst,
                            double* gx) {
    for (int64_t i = 0; i < n_dst; i++) {
        int64_t deg = offsets[i + 1] - offsets[i];
        for (int64_t e = offsets[i]; e < offsets[i + 1]; e++)
            for (int64_t c = 0; c < dim; c++) gx[(int64_t)src[e] * dim + c] += g[i * dim + c] / (double)deg;
    }
}
