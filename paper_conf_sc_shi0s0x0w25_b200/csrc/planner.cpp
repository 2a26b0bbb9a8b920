// planner.cpp — host planner of the Moment hot path: topology graph (P1), Dinic rate max-flow (P3),
// DDAK placement (P4), time-bisection ingest plan + quotas (P5). Citations: PAPER.md lines "P:Lnnn";
// readings R# are DESIGN.md §3. Offline, host-only, deterministic.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <limits>
#include <mutex>
#include <new>
#include <thread>
#include <vector>

#include "moment.h"
#include "status.h"

namespace moment {

static thread_local std::string g_err;
void set_error(const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_err = buf;
}
const char* last_error() { return g_err.c_str(); }

static constexpr int64_t kInf = MOMENT_CAP_INF;
static constexpr int64_t kScaledLimit = int64_t(1) << 62;  // finite ceiling of cap * T (R10)

// ---------------------------------------------------------------------------------------------
// Dinic max-flow with INF capacities. Arc 2i / 2i+1 = link i forward / backward.
// ---------------------------------------------------------------------------------------------
class Dinic {
  public:
    Dinic(int n, const std::vector<int32_t>& from, const std::vector<int32_t>& to, const std::vector<int64_t>& cap)
        : n_(n), from_(from), to_(to), head_(n, -1), level_(n), it_(n) {
        const size_t m = from.size();
        res_.resize(2 * m);
        next_.resize(2 * m);
        // Build adjacency lists so that iteration visits arcs in link order (insert in reverse).
        for (size_t ii = m; ii-- > 0;) {
            res_[2 * ii] = cap[ii];
            res_[2 * ii + 1] = 0;
            push_arc(from[ii], int64_t(2 * ii));
            push_arc(to[ii], int64_t(2 * ii + 1));
        }
    }

    // Returns MOMENT_OK and the flow value, EINVAL when unbounded, EOVERFLOW on int64 overflow.
    moment_status run(int s, int t, int64_t* value) {
        if (inf_path(s, t)) return fail(MOMENT_EINVAL, "max-flow is unbounded: an s-t path of INF links exists");
        int64_t total = 0;
        while (bfs(s, t)) {
            for (int u = 0; u < n_; u++) it_[u] = head_[u];
            for (;;) {
                int64_t f = dfs(s, t, kInf);
                if (f == 0) break;
                if (f == kInf) return fail(MOMENT_EINVAL, "max-flow is unbounded");
                if (__builtin_add_overflow(total, f, &total) || total == kInf)
                    return fail(MOMENT_EOVERFLOW, "max-flow value overflows int64");
            }
        }
        *value = total;
        return MOMENT_OK;
    }

    int64_t flow(size_t link) const { return res_[2 * link + 1]; }

    // Nodes reachable from s in the residual graph (min-cut side S).
    std::vector<char> reachable(int s) const {
        std::vector<char> seen(n_, 0);
        std::vector<int> st{s};
        seen[s] = 1;
        while (!st.empty()) {
            int u = st.back();
            st.pop_back();
            for (int64_t a = head_[u]; a >= 0; a = next_[a]) {
                int w = other(a);
                if (!seen[w] && res_[a] > 0) { seen[w] = 1; st.push_back(w); }
            }
        }
        return seen;
    }

  private:
    void push_arc(int u, int64_t a) {
        next_[a] = head_[u];
        head_[u] = a;
    }
    int other(int64_t a) const { return (a & 1) ? from_[a >> 1] : to_[a >> 1]; }

    bool inf_path(int s, int t) const {
        std::vector<char> seen(n_, 0);
        std::vector<int> st{s};
        seen[s] = 1;
        while (!st.empty()) {
            int u = st.back();
            st.pop_back();
            for (int64_t a = head_[u]; a >= 0; a = next_[a]) {
                if ((a & 1) || res_[a] != kInf) continue;
                int w = to_[a >> 1];
                if (!seen[w]) { seen[w] = 1; st.push_back(w); }
            }
        }
        return seen[t];
    }

    bool bfs(int s, int t) {
        std::fill(level_.begin(), level_.end(), -1);
        std::vector<int> q;
        q.reserve(n_);
        q.push_back(s);
        level_[s] = 0;
        for (size_t qi = 0; qi < q.size(); qi++) {
            int u = q[qi];
            for (int64_t a = head_[u]; a >= 0; a = next_[a]) {
                int w = other(a);
                if (level_[w] < 0 && res_[a] > 0) {
                    level_[w] = level_[u] + 1;
                    q.push_back(w);
                }
            }
        }
        return level_[t] >= 0;
    }

    int64_t dfs(int u, int t, int64_t limit) {
        if (u == t) return limit;
        for (int64_t& a = it_[u]; a >= 0; a = next_[a]) {
            int w = other(a);
            if (res_[a] <= 0 || level_[w] != level_[u] + 1) continue;
            int64_t pushed = dfs(w, t, std::min(limit, res_[a]));
            if (pushed > 0) {
                if (pushed != kInf) {
                    if (res_[a] != kInf) res_[a] -= pushed;
                    int64_t& back = res_[a ^ 1];
                    if (back != kInf) back += pushed;
                }
                return pushed;
            }
        }
        return 0;
    }

    int n_;
    std::vector<int32_t> from_, to_;
    std::vector<int64_t> head_, next_, res_;
    std::vector<int> level_;
    std::vector<int64_t> it_;
};

}  // namespace moment

using namespace moment;

// ---------------------------------------------------------------------------------------------
// P1 — topology
// ---------------------------------------------------------------------------------------------
struct moment_topo_s {
    std::vector<moment_node> nodes;
    std::vector<moment_link> links;
    int32_t s = -1, t = -1;
};

static bool link_allowed(int32_t fk, int32_t tk) {
    // source -> storage -> interconnect -> computation -> sink; storage may feed a GPU directly.
    switch (fk) {
        case MOMENT_NODE_SOURCE: return tk == MOMENT_NODE_STORAGE;
        case MOMENT_NODE_STORAGE: return tk == MOMENT_NODE_INTERCONNECT || tk == MOMENT_NODE_COMPUTE;
        case MOMENT_NODE_INTERCONNECT: return tk == MOMENT_NODE_INTERCONNECT || tk == MOMENT_NODE_COMPUTE;
        case MOMENT_NODE_COMPUTE: return tk == MOMENT_NODE_SINK;
        default: return false;
    }
}

extern "C" moment_status moment_topology(const moment_node* nodes, int32_t n_nodes, const moment_link* links,
                                         int32_t n_links, moment_topo_t* out) {
    if (!out || n_nodes <= 0 || n_links < 0 || !nodes || (n_links > 0 && !links))
        return fail(MOMENT_EINVAL, "moment_topology: null argument or non-positive size");
    *out = nullptr;
    auto* T = new (std::nothrow) moment_topo_s;
    if (!T) return fail(MOMENT_ENOMEM, "moment_topology: out of host memory");
    T->nodes.assign(nodes, nodes + n_nodes);
    T->links.assign(links, links + n_links);
    auto bad = [&](const char* fmt, int64_t a, int64_t b) {
        delete T;
        return fail(MOMENT_EINVAL, fmt, (long long)a, (long long)b);
    };
    for (int32_t v = 0; v < n_nodes; v++) {
        const moment_node& nd = nodes[v];
        if (nd.kind < MOMENT_NODE_SOURCE || nd.kind > MOMENT_NODE_COMPUTE || nd.reserved != 0)
            return bad("moment_topology: node %lld has invalid kind %lld", v, nd.kind);
        if (nd.kind == MOMENT_NODE_STORAGE && (nd.tier < MOMENT_TIER_GPU_HBM || nd.tier > MOMENT_TIER_SSD))
            return bad("moment_topology: storage node %lld has invalid tier %lld", v, nd.tier);
        if (nd.kind == MOMENT_NODE_SOURCE) {
            if (T->s >= 0) return bad("moment_topology: two source nodes (%lld, %lld)", T->s, v);
            T->s = v;
        }
        if (nd.kind == MOMENT_NODE_SINK) {
            if (T->t >= 0) return bad("moment_topology: two sink nodes (%lld, %lld)", T->t, v);
            T->t = v;
        }
    }
    for (int32_t i = 0; i < n_links; i++) {
        const moment_link& l = links[i];
        if (l.from < 0 || l.from >= n_nodes || l.to < 0 || l.to >= n_nodes)
            return bad("moment_topology: link %lld references node %lld out of range", i,
                       (l.from < 0 || l.from >= n_nodes) ? l.from : l.to);
        if (l.from == l.to) return bad("moment_topology: link %lld is a self-loop at node %lld", i, l.from);
        if (l.cap < 0) return bad("moment_topology: link %lld has negative capacity %lld", i, l.cap);
        if (!link_allowed(nodes[l.from].kind, nodes[l.to].kind))
            return bad("moment_topology: link %lld direction kind %lld -> not allowed (P:L215)", i,
                       nodes[l.from].kind);
    }
    if (T->s < 0) {
        T->s = (int32_t)T->nodes.size();
        T->nodes.push_back({MOMENT_NODE_SOURCE, MOMENT_TIER_NONE, -1, 0});
    }
    if (T->t < 0) {
        T->t = (int32_t)T->nodes.size();
        T->nodes.push_back({MOMENT_NODE_SINK, MOMENT_TIER_NONE, -1, 0});
    }
    const int32_t N = (int32_t)T->nodes.size();
    std::vector<char> has_src(N, 0), has_sink(N, 0);
    std::vector<int64_t> out_cap(N, 0);
    for (const auto& l : T->links) {
        if (l.from == T->s) has_src[l.to] = 1;
        if (l.to == T->t) has_sink[l.from] = 1;
        if (T->nodes[l.from].kind == MOMENT_NODE_STORAGE) {
            int64_t& c = out_cap[l.from];
            if (c == kInf || l.cap == kInf || __builtin_add_overflow(c, l.cap, &c)) c = kInf;
        }
    }
    // c(s, v_s) = c(v_s, v_i) (R8): the storage node's total egress capacity.
    for (int32_t v = 0; v < N; v++)
        if (T->nodes[v].kind == MOMENT_NODE_STORAGE && !has_src[v]) T->links.push_back({T->s, v, out_cap[v]});
    for (int32_t v = 0; v < N; v++)
        if (T->nodes[v].kind == MOMENT_NODE_COMPUTE && !has_sink[v]) T->links.push_back({v, T->t, kInf});
    *out = T;
    return MOMENT_OK;
}

extern "C" moment_status moment_topology_info(moment_topo_t T, int32_t* n_nodes, int32_t* n_links, int32_t* source,
                                              int32_t* sink) {
    if (!T) return fail(MOMENT_EINVAL, "moment_topology_info: null topology");
    if (n_nodes) *n_nodes = (int32_t)T->nodes.size();
    if (n_links) *n_links = (int32_t)T->links.size();
    if (source) *source = T->s;
    if (sink) *sink = T->t;
    return MOMENT_OK;
}

extern "C" moment_status moment_topology_export(moment_topo_t T, moment_node* nodes, moment_link* links) {
    if (!T) return fail(MOMENT_EINVAL, "moment_topology_export: null topology");
    if (nodes) std::memcpy(nodes, T->nodes.data(), T->nodes.size() * sizeof(moment_node));
    if (links) std::memcpy(links, T->links.data(), T->links.size() * sizeof(moment_link));
    return MOMENT_OK;
}

extern "C" moment_status moment_topology_free(moment_topo_t T) {
    delete T;
    return MOMENT_OK;
}

// ---------------------------------------------------------------------------------------------
// P3 — rate max-flow
// ---------------------------------------------------------------------------------------------
static moment_status run_flow(int n, const std::vector<int32_t>& from, const std::vector<int32_t>& to,
                              const std::vector<int64_t>& cap, int s, int t, int64_t* value,
                              std::vector<int64_t>* flow) {
    Dinic d(n, from, to, cap);
    MOMENT_TRY(d.run(s, t, value));
    if (flow) {
        flow->resize(from.size());
        for (size_t i = 0; i < from.size(); i++) (*flow)[i] = d.flow(i);
    }
    return MOMENT_OK;
}

static void split_links(const moment_topo_s* T, std::vector<int32_t>& from, std::vector<int32_t>& to,
                        std::vector<int64_t>& cap) {
    from.resize(T->links.size());
    to.resize(T->links.size());
    cap.resize(T->links.size());
    for (size_t i = 0; i < T->links.size(); i++) {
        from[i] = T->links[i].from;
        to[i] = T->links[i].to;
        cap[i] = T->links[i].cap;
    }
}

extern "C" moment_status moment_maxflow(moment_topo_t T, int64_t* value, int64_t* link_flow) {
    if (!T || !value) return fail(MOMENT_EINVAL, "moment_maxflow: null argument");
    std::vector<int32_t> from, to;
    std::vector<int64_t> cap, flow;
    split_links(T, from, to, cap);
    MOMENT_TRY(run_flow((int)T->nodes.size(), from, to, cap, T->s, T->t, value, &flow));
    if (link_flow) std::memcpy(link_flow, flow.data(), flow.size() * sizeof(int64_t));
    return MOMENT_OK;
}

// ---------------------------------------------------------------------------------------------
// P4 — DDAK
// ---------------------------------------------------------------------------------------------
namespace {

using u128 = unsigned __int128;

// Compare p1/q1 with p2/q2 (q > 0) exactly by continued-fraction expansion; no 256-bit products.
int cmp_frac(u128 p1, u128 q1, u128 p2, u128 q2) {
    int sign = 1;  // +1 while comparing x = p1/q1 with y = p2/q2 directly, -1 once reversed
    for (;;) {
        u128 a1 = p1 / q1, a2 = p2 / q2;
        if (a1 != a2) return a1 < a2 ? -sign : sign;
        u128 r1 = p1 % q1, r2 = p2 % q2;
        if (r1 == 0 && r2 == 0) return 0;
        if (r1 == 0) return -sign;  // x = a < a + r2/q2 = y
        if (r2 == 0) return sign;
        // r1/q1 < r2/q2  <=>  q1/r1 > q2/r2: continue on the reciprocals with the order flipped
        u128 np1 = q1, nq1 = r1, np2 = q2, nq2 = r2;
        p1 = np1; q1 = nq1; p2 = np2; q2 = nq2;
        sign = -sign;
    }
}

struct Bin {
    uint64_t access = 0;  // A: cumulative hotness
    uint64_t demand = 0;  // A': cumulative demand counts (replication search only)
    int64_t used = 0;     // U: rows placed
    int64_t cap = 0;      // C
    int64_t traffic = 0;  // T
    int32_t rank = 0;     // tier rank (0 best)
};

// -1 if priority(a) < priority(b); Eq. 2 priority = (A/T)(U/C), T = 0 => +inf.
int priority_cmp(const Bin& a, const Bin& b) {
    bool ia = a.traffic == 0, ib = b.traffic == 0;
    if (ia || ib) return ia && ib ? 0 : (ia ? 1 : -1);
    u128 pa = (u128)a.access * (u128)(uint64_t)a.used, qa = (u128)(uint64_t)a.traffic * (u128)(uint64_t)a.cap;
    u128 pb = (u128)b.access * (u128)(uint64_t)b.used, qb = (u128)(uint64_t)b.traffic * (u128)(uint64_t)b.cap;
    return cmp_frac(pa, qa, pb, qb);
}

// -1 if a is less filled than b (U_a / C_a < U_b / C_b), exactly; C > 0 for non-full bins.
int fill_cmp(const Bin& a, const Bin& b) {
    const u128 l = (u128)(uint64_t)a.used * (u128)(uint64_t)b.cap, r = (u128)(uint64_t)b.used * (u128)(uint64_t)a.cap;
    return l < r ? -1 : (l > r ? 1 : 0);
}

// Stable LSD radix sort of vertex ids by descending hotness (ties: ascending id, from stability).
void order_by_hotness(int64_t n, const uint64_t* hot, std::vector<uint32_t>& order) {
    order.resize(n);
    std::vector<uint32_t> tmp(n);
    for (int64_t i = 0; i < n; i++) order[i] = (uint32_t)i;
    unsigned nthreads = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
    if (n < (1 << 20)) nthreads = 1;
    for (int pass = 0; pass < 8; pass++) {
        const int shift = 8 * pass;
        std::vector<std::vector<int64_t>> hist(nthreads, std::vector<int64_t>(256, 0));
        auto chunk = [&](unsigned t, int64_t& lo, int64_t& hi) {
            lo = n * t / nthreads;
            hi = n * (t + 1) / nthreads;
        };
        auto count = [&](unsigned t) {
            int64_t lo, hi;
            chunk(t, lo, hi);
            auto& h = hist[t];
            for (int64_t i = lo; i < hi; i++) h[255 - ((hot[order[i]] >> shift) & 0xFF)]++;
        };
        std::vector<std::thread> th;
        for (unsigned t = 1; t < nthreads; t++) th.emplace_back(count, t);
        count(0);
        for (auto& x : th) x.join();
        th.clear();
        int nonempty = 0;
        for (int b = 0; b < 256; b++) {
            int64_t tot = 0;
            for (unsigned t = 0; t < nthreads; t++) tot += hist[t][b];
            nonempty += tot > 0;
        }
        if (nonempty <= 1) continue;  // every key has the same byte: the pass is the identity
        int64_t base = 0;
        for (int b = 0; b < 256; b++)
            for (unsigned t = 0; t < nthreads; t++) {
                int64_t c = hist[t][b];
                hist[t][b] = base;
                base += c;
            }
        auto scatter = [&](unsigned t) {
            int64_t lo, hi;
            chunk(t, lo, hi);
            auto& h = hist[t];
            for (int64_t i = lo; i < hi; i++) {
                uint32_t v = order[i];
                tmp[h[255 - ((hot[v] >> shift) & 0xFF)]++] = v;
            }
        };
        for (unsigned t = 1; t < nthreads; t++) th.emplace_back(scatter, t);
        scatter(0);
        for (auto& x : th) x.join();
        order.swap(tmp);
    }
}

uint64_t mix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

// Bins of a placement call: node, tier rank, capacity and Bin_traffic resolved from args/topology.
moment_status resolve_bins(moment_topo_t T, const moment_place_args* a, std::vector<Bin>& bins,
                           std::vector<int32_t>& bin_node) {
    const int32_t nb = a->n_bins;
    if (nb <= 0 || nb > MOMENT_MAX_BINS) return fail(MOMENT_EINVAL, "moment_place: n_bins %d out of range", nb);
    if (!a->bin_capacity_rows) return fail(MOMENT_EINVAL, "moment_place: bin_capacity_rows is null");
    bin_node.assign(nb, -1);
    if (a->bin_node) {
        for (int b = 0; b < nb; b++) bin_node[b] = a->bin_node[b];
    } else if (T) {
        int b = 0;
        for (int32_t v = 0; v < (int32_t)T->nodes.size() && b < nb; v++)
            if (T->nodes[v].kind == MOMENT_NODE_STORAGE) bin_node[b++] = v;
        if (b != nb) return fail(MOMENT_EINVAL, "moment_place: topology has %d storage nodes, n_bins = %d", b, nb);
    }
    bins.assign(nb, Bin{});
    std::vector<int64_t> traffic(nb, 0);
    if (a->bin_traffic) {
        for (int b = 0; b < nb; b++) traffic[b] = a->bin_traffic[b];
    } else {
        if (!T) return fail(MOMENT_EINVAL, "moment_place: bin_traffic is null and no topology given");
        if (a->traffic_mode != MOMENT_TRAFFIC_RATE_FLOW && a->traffic_mode != MOMENT_TRAFFIC_STANDALONE)
            return fail(MOMENT_EINVAL, "moment_place: unknown traffic_mode %d", a->traffic_mode);
        std::vector<int32_t> from, to;
        std::vector<int64_t> cap, flow;
        split_links(T, from, to, cap);
        for (int b = 0; b < nb; b++)
            if (bin_node[b] < 0) return fail(MOMENT_EINVAL, "moment_place: bin %d has no topology node", b);
        int64_t F = 0;
        if (a->traffic_mode == MOMENT_TRAFFIC_RATE_FLOW) {
            MOMENT_TRY(run_flow((int)T->nodes.size(), from, to, cap, T->s, T->t, &F, &flow));
            for (int b = 0; b < nb; b++)
                for (size_t i = 0; i < T->links.size(); i++)
                    if (T->links[i].from == T->s && T->links[i].to == bin_node[b]) traffic[b] += flow[i];
        } else {
            for (int b = 0; b < nb; b++) {
                std::vector<int64_t> c = cap;
                for (size_t i = 0; i < T->links.size(); i++)
                    if (T->links[i].from == T->s && T->links[i].to != bin_node[b]) c[i] = 0;
                MOMENT_TRY(run_flow((int)T->nodes.size(), from, to, c, T->s, T->t, &F, nullptr));
                traffic[b] = F;
            }
        }
    }
    for (int b = 0; b < nb; b++) {
        int32_t tier;
        if (a->bin_tier) tier = a->bin_tier[b];
        else if (T && bin_node[b] >= 0 && bin_node[b] < (int32_t)T->nodes.size()) tier = T->nodes[bin_node[b]].tier;
        else return fail(MOMENT_EINVAL, "moment_place: no tier for bin %d", b);
        if (tier < MOMENT_TIER_GPU_HBM || tier > MOMENT_TIER_SSD) return fail(MOMENT_EINVAL, "moment_place: bin %d tier %d", b, tier);
        if (a->bin_capacity_rows[b] < 0 || traffic[b] < 0) return fail(MOMENT_EINVAL, "moment_place: bin %d negative capacity/traffic", b);
        bins[b].rank = tier - 1;
        bins[b].cap = a->bin_capacity_rows[b];
        bins[b].traffic = traffic[b];
    }
    return MOMENT_OK;
}

// DDAK over `order` (hotness desc, id asc) with the first r vertices replicated in every GPU bin (R25;
// r = 0: plain DDAK, R13-R17). bin_of/slot_of may be null (the search needs only A, U per bin).
moment_status ddak_core(int64_t n, const uint64_t* hot, const std::vector<uint32_t>& order, int64_t r, int64_t pool,
                        std::vector<Bin>& bins, uint64_t* replica_access, int32_t* bin_of, int64_t* slot_of,
                        const uint64_t* dem = nullptr, uint64_t* replica_demand = nullptr) {
    const int nb = (int)bins.size();
    if (r < 0 || r > n) return fail(MOMENT_EINVAL, "moment_place: replicate_rows %lld out of [0, %lld]", (long long)r, (long long)n);
    std::vector<int64_t> slot0(nb, 0);
    int64_t total_cap = 0;
    for (int b = 0; b < nb; b++) {
        if (r > 0 && bins[b].rank == MOMENT_TIER_GPU_HBM - 1) {
            if (bins[b].cap < r)
                return fail(MOMENT_EINFEASIBLE, "moment_place: replicate_rows %lld exceeds GPU bin %d capacity %lld",
                            (long long)r, b, (long long)bins[b].cap);
            bins[b].cap -= r;  // Eq. 2 runs on the residual capacity; the partition's slots start at r
            slot0[b] = r;
        }
        total_cap += bins[b].cap;
    }
    if (total_cap < n - r)
        return fail(MOMENT_EINFEASIBLE, "moment_place: capacity %lld rows < %lld vertices", (long long)total_cap, (long long)(n - r));
    uint64_t rep = 0, rep_dem = 0;
    for (int64_t i = 0; i < r; i++) {
        const uint32_t v = order[i];
        if (bin_of) { bin_of[v] = MOMENT_BIN_REPLICA; slot_of[v] = i; }
        rep += hot[v];
        if (dem) rep_dem += dem[v];
    }
    if (replica_access) *replica_access = rep;
    if (replica_demand) *replica_demand = rep_dem;
    for (int64_t g0 = r; g0 < n; g0 += pool) {
        int64_t next = g0, g1 = std::min(n, g0 + pool);
        while (next < g1) {
            int best_rank = std::numeric_limits<int>::max();
            for (auto& b : bins)
                if (b.used < b.cap && b.traffic > 0) best_rank = std::min(best_rank, b.rank);
            int pick = -1;
            for (int b = 0; b < nb; b++) {
                const Bin& B = bins[b];
                if (B.used >= B.cap) continue;
                if (best_rank != std::numeric_limits<int>::max() && B.rank != best_rank) continue;
                if (pick < 0) { pick = b; continue; }
                int c = priority_cmp(B, bins[pick]);
                if (c == 0) c = fill_cmp(B, bins[pick]);  // R16: equal priority -> the less-filled bin
                if (c < 0 || (c == 0 && B.rank < bins[pick].rank)) pick = b;
            }
            if (pick < 0) return fail(MOMENT_EINFEASIBLE, "moment_place: no bin has room");
            Bin& B = bins[pick];
            int64_t m = std::min(g1 - next, B.cap - B.used);
            uint64_t acc = 0, dacc = 0;
            for (int64_t q = 0; q < m; q++) {
                uint32_t v = order[next + q];
                if (bin_of) { bin_of[v] = pick; slot_of[v] = slot0[pick] + B.used + q; }
                acc += hot[v];
                if (dem) dacc += dem[v];
            }
            B.access += acc;
            B.demand += dacc;
            B.used += m;
            next += m;
        }
    }
    return MOMENT_OK;
}

}  // namespace

extern "C" moment_status moment_place(moment_topo_t T, const moment_place_args* a, moment_place_out* o) {
    if (!a || !o || !o->bin_of || !o->slot_of) return fail(MOMENT_EINVAL, "moment_place: null argument");
    const int64_t n = a->n_vertices;
    const int32_t nb = a->n_bins;
    if (n < 0 || n >= (int64_t(1) << 32)) return fail(MOMENT_EINVAL, "moment_place: n_vertices %lld out of range", (long long)n);
    if (n > 0 && !a->hotness && a->mode == MOMENT_PLACE_DDAK) return fail(MOMENT_EINVAL, "moment_place: hotness is null");
    std::vector<Bin> bins;
    std::vector<int32_t> bin_node;
    MOMENT_TRY(resolve_bins(T, a, bins, bin_node));
    if (o->replica_access) *o->replica_access = 0;
    if (a->mode == MOMENT_PLACE_HASH) {
        if (a->replicate_rows != 0) return fail(MOMENT_EINVAL, "moment_place: replicate_rows needs DDAK mode");
        int64_t total_cap = 0;
        for (auto& b : bins) total_cap += b.cap;
        if (total_cap < n) return fail(MOMENT_EINFEASIBLE, "moment_place: capacity %lld rows < %lld vertices", (long long)total_cap, (long long)n);
        // Uniform baseline ("hash-based partitioning"): bin = hash(v) mod n_bins, next non-full
        // bin on overflow; slots in id order.
        for (int64_t v = 0; v < n; v++) {
            int b = (int)(mix64((uint64_t)v) % (uint64_t)nb);
            while (bins[b].used >= bins[b].cap) b = (b + 1) % nb;
            o->bin_of[v] = b;
            o->slot_of[v] = bins[b].used++;
            bins[b].access += a->hotness ? a->hotness[v] : 0;
        }
    } else if (a->mode == MOMENT_PLACE_DDAK) {
        std::vector<uint32_t> order;
        order_by_hotness(n, a->hotness, order);
        const int64_t pool = a->pool > 0 ? a->pool : 100;
        MOMENT_TRY(ddak_core(n, a->hotness, order, a->replicate_rows, pool, bins, o->replica_access, o->bin_of,
                             o->slot_of));
    } else {
        return fail(MOMENT_EINVAL, "moment_place: unknown mode %d", a->mode);
    }
    for (int b = 0; b < nb; b++) {
        if (o->bin_access) o->bin_access[b] = bins[b].access;
        if (o->bin_rows_used) o->bin_rows_used[b] = bins[b].used;
        if (o->bin_traffic_used) o->bin_traffic_used[b] = bins[b].traffic;
    }
    return MOMENT_OK;
}

extern "C" moment_status moment_place_pack_rank(int64_t n, const int32_t* bin_of, const int64_t* slot_of,
                                               int32_t replica_bin, uint64_t* packed) {
    if (n < 0 || (n > 0 && (!bin_of || !slot_of || !packed))) return fail(MOMENT_EINVAL, "moment_place_pack_rank: null argument");
    if (replica_bin < 0 || replica_bin >= MOMENT_MAX_BINS)
        return fail(MOMENT_EINVAL, "moment_place_pack_rank: replica_bin %d out of range", replica_bin);
    for (int64_t v = 0; v < n; v++) {
        const int32_t b = bin_of[v] == MOMENT_BIN_REPLICA ? replica_bin : bin_of[v];
        if (b < 0 || b >= MOMENT_MAX_BINS || slot_of[v] < 0 || slot_of[v] >= (int64_t(1) << 40))
            return fail(MOMENT_EINVAL, "moment_place_pack_rank: vertex %lld has bin %d slot %lld out of range", (long long)v,
                        bin_of[v], (long long)slot_of[v]);
        packed[v] = ((uint64_t)b << 40) | (uint64_t)slot_of[v];
    }
    return MOMENT_OK;
}

extern "C" moment_status moment_place_pack(int64_t n, const int32_t* bin_of, const int64_t* slot_of, uint64_t* packed) {
    if (n < 0 || (n > 0 && (!bin_of || !slot_of || !packed))) return fail(MOMENT_EINVAL, "moment_place_pack: null argument");
    for (int64_t v = 0; v < n; v++) {
        if (bin_of[v] < 0 || bin_of[v] >= MOMENT_MAX_BINS || slot_of[v] < 0 || slot_of[v] >= (int64_t(1) << 40))
            return fail(MOMENT_EINVAL, "moment_place_pack: vertex %lld has bin %d slot %lld out of range", (long long)v,
                        bin_of[v], (long long)slot_of[v]);
        packed[v] = ((uint64_t)bin_of[v] << 40) | (uint64_t)slot_of[v];
    }
    return MOMENT_OK;
}

// ---------------------------------------------------------------------------------------------
// P5 — time-bisection ingest plan and quotas (R10-R12)
// ---------------------------------------------------------------------------------------------
struct moment_plan_s {
    int32_t k = 0, n_nodes = 0;
    int64_t t_star = 0, t_ingest = 0, t_nvlink = 0, t_hbm = 0;
    std::vector<int64_t> link_flow;  // ingest flow at T_ingest
    std::vector<int64_t> quota;      // [n_nodes][k]
};

namespace {

struct Ingest {
    int n = 0, s = -1, t = -1;
    std::vector<int32_t> from, to;
    std::vector<int64_t> cap;
    std::vector<char> supply;
};

moment_status flow_at_time(const Ingest& G, int64_t T, int64_t* value, std::vector<int64_t>* flow) {
    std::vector<int64_t> c(G.cap.size());
    for (size_t i = 0; i < c.size(); i++) {
        if (G.supply[i] || G.cap[i] == kInf) c[i] = G.cap[i];
        else if (T < 0) c[i] = G.cap[i] == 0 ? 0 : kInf;  // reachability: a closed link stays closed
        else if (G.cap[i] != 0 && T > kScaledLimit / G.cap[i]) c[i] = kScaledLimit;
        else c[i] = G.cap[i] * T;
    }
    return run_flow(G.n, G.from, G.to, c, G.s, G.t, value, flow);
}

int64_t ceil_div(u128 a, u128 b) { return (int64_t)((a + b - 1) / b); }

}  // namespace

extern "C" moment_status moment_plan(moment_topo_t T, const moment_plan_args* a, moment_plan_t* out) {
    if (!T || !a || !out || !a->gpu_node || !a->bin_demand_bytes) return fail(MOMENT_EINVAL, "moment_plan: null argument");
    *out = nullptr;
    const int k = a->k;
    const int N = (int)T->nodes.size();
    if (k <= 0 || k > 1024) return fail(MOMENT_EINVAL, "moment_plan: k = %d out of range", k);
    std::vector<int> rank_of_node(N, -1), rank_of_device;
    for (int r = 0; r < k; r++) {
        int v = a->gpu_node[r];
        if (v < 0 || v >= N || T->nodes[v].kind != MOMENT_NODE_COMPUTE || rank_of_node[v] >= 0)
            return fail(MOMENT_EINVAL, "moment_plan: gpu_node[%d] = %d is not a distinct compute node", r, v);
        rank_of_node[v] = r;
    }
    auto owner_rank = [&](int v) -> int {  // rank of the active GPU whose device owns HBM node v
        for (int r = 0; r < k; r++)
            if (T->nodes[a->gpu_node[r]].device == T->nodes[v].device) return r;
        return -1;
    };
    for (int v = 0; v < N; v++)
        if (T->nodes[v].kind == MOMENT_NODE_STORAGE && a->bin_demand_bytes[v] < 0)
            return fail(MOMENT_EINVAL, "moment_plan: negative demand on node %d", v);
    Ingest G;
    G.n = N;
    G.s = T->s;
    G.t = T->t;
    for (const auto& l : T->links) {
        int64_t c = l.cap;
        char sup = 0;
        if (l.from == T->s) {
            const moment_node& nd = T->nodes[l.to];
            sup = 1;
            if (nd.tier == MOMENT_TIER_GPU_HBM) c = 0;
            else {
                u128 d = (u128)k * (u128)a->bin_demand_bytes[l.to];
                if (d > (u128)kScaledLimit) return fail(MOMENT_EOVERFLOW, "moment_plan: demand overflows");
                c = (int64_t)d;
            }
        } else if (l.to == T->t) {
            c = rank_of_node[l.from] >= 0 ? kInf : 0;
        }
        G.from.push_back(l.from);
        G.to.push_back(l.to);
        G.cap.push_back(c);
        G.supply.push_back(sup);
    }
    int64_t D = 0;
    for (size_t i = 0; i < G.cap.size(); i++)
        if (G.supply[i]) D += G.cap[i];
    auto* P = new (std::nothrow) moment_plan_s;
    if (!P) return fail(MOMENT_ENOMEM, "moment_plan: out of memory");
    P->k = k;
    P->n_nodes = N;
    int64_t v = 0;
    // T_ingest: doubling then bisection on the monotone predicate maxflow(T) == D.
    int64_t Tlo = 0, Thi = 0;
    if (D > 0) {
        moment_status st = flow_at_time(G, -1, &v, nullptr);
        if (st != MOMENT_OK) { delete P; return st; }
        if (v < D) { delete P; return fail(MOMENT_EINFEASIBLE, "moment_plan: demand %lld unreachable (max %lld)", (long long)D, (long long)v); }
        Thi = 1;
        for (;;) {
            st = flow_at_time(G, Thi, &v, nullptr);
            if (st != MOMENT_OK) { delete P; return st; }
            if (v == D) break;
            if (Thi > (int64_t(1) << 61)) { delete P; return fail(MOMENT_EINFEASIBLE, "moment_plan: no finite T"); }
            Tlo = Thi;
            Thi *= 2;
        }
        while (Thi - Tlo > 1) {
            int64_t mid = Tlo + (Thi - Tlo) / 2;
            st = flow_at_time(G, mid, &v, nullptr);
            if (st != MOMENT_OK) { delete P; return st; }
            (v == D ? Thi : Tlo) = mid;
        }
    }
    P->t_ingest = Thi;
    moment_status st = flow_at_time(G, Thi, &v, &P->link_flow);
    if (st != MOMENT_OK) { delete P; return st; }
    // x[j][h]: walk the flow from each host bin j to a computation node, cancelling cycles.
    P->quota.assign((size_t)N * k, 0);
    std::vector<int64_t> rem = P->link_flow;
    std::vector<std::vector<int>> out_links(N);
    for (size_t i = 0; i < G.from.size(); i++) out_links[G.from[i]].push_back((int)i);
    for (size_t i = 0; i < G.from.size(); i++) {
        if (!(G.supply[i] && rem[i] > 0)) continue;
        const int j = G.to[i];
        while (rem[i] > 0) {
            std::vector<int> path;  // link indices from j
            std::vector<int> pos(N, -1);
            int u = j;
            pos[u] = 0;
            for (;;) {
                if (rank_of_node[u] >= 0) {
                    // computation node: terminate on its sink link
                    int tl = -1;
                    for (int li : out_links[u])
                        if (G.to[li] == G.t && rem[li] > 0) { tl = li; break; }
                    if (tl >= 0) { path.push_back(tl); break; }
                }
                int nxt = -1;
                for (int li : out_links[u])
                    if (rem[li] > 0 && G.to[li] != G.t) { nxt = li; break; }
                if (nxt < 0) { delete P; return fail(MOMENT_EINVAL, "moment_plan: flow decomposition stuck at node %d", u); }
                int w = G.to[nxt];
                if (pos[w] >= 0) {  // cycle: cancel it and resume from w
                    int64_t m = rem[nxt];
                    for (size_t q = pos[w]; q < path.size(); q++) m = std::min(m, rem[path[q]]);
                    rem[nxt] -= m;
                    for (size_t q = pos[w]; q < path.size(); q++) rem[path[q]] -= m;
                    for (size_t q = pos[w]; q < path.size(); q++) pos[G.to[path[q]]] = -1;
                    path.resize(pos[w]);
                    pos[w] = (int)path.size();
                    u = w;
                    continue;
                }
                path.push_back(nxt);
                pos[w] = (int)path.size();
                u = w;
            }
            int64_t m = rem[i];
            for (int li : path) m = std::min(m, rem[li]);
            rem[i] -= m;
            for (int li : path) rem[li] -= m;
            P->quota[(size_t)j * k + rank_of_node[G.from[path.back()]]] += m;
        }
    }
    // Closed forms (R11).
    if (a->replica_demand_bytes < 0) { delete P; return fail(MOMENT_EINVAL, "moment_plan: negative replica demand"); }
    // every GPU writes its whole batch: partitioned demand + the replicated rows, which it also reads
    // from its own HBM (R25)
    int64_t total_d = 2 * a->replica_demand_bytes;
    for (int b = 0; b < N; b++)
        if (T->nodes[b].kind == MOMENT_NODE_STORAGE) total_d += a->bin_demand_bytes[b];
    int64_t max_link = 0, max_hbm = 0;
    for (int g = 0; g < k; g++) {
        int64_t in_g = 0, out_g = 0, hbm_g = total_d;
        for (int b = 0; b < N; b++) {
            const moment_node& nd = T->nodes[b];
            if (nd.kind != MOMENT_NODE_STORAGE) continue;
            const int64_t d = a->bin_demand_bytes[b];
            if (nd.tier == MOMENT_TIER_GPU_HBM) {
                int o = owner_rank(b);
                if (o < 0) {
                    if (d > 0) { delete P; return fail(MOMENT_EINVAL, "moment_plan: HBM node %d has demand but no active owner", b); }
                    continue;
                }
                if (o == g) { out_g += (int64_t)(k - 1) * d; hbm_g += (int64_t)k * d; }
                else in_g += d;
            } else {
                int64_t W = 0;
                for (int h = 0; h < k; h++) W += P->quota[(size_t)b * k + h];
                if (W == 0 || d == 0) continue;
                const int64_t xg = P->quota[(size_t)b * k + g];
                in_g += ceil_div((u128)d * (u128)(W - xg), (u128)W);
                out_g += ceil_div((u128)(k - 1) * (u128)d * (u128)xg, (u128)W);
            }
        }
        max_link = std::max(max_link, std::max(in_g, out_g));
        max_hbm = std::max(max_hbm, hbm_g);
    }
    if (max_link > 0 && a->nvlink_cap <= 0) { delete P; return fail(MOMENT_EINFEASIBLE, "moment_plan: peer traffic but nvlink_cap = 0"); }
    if (a->hbm_cap <= 0) { delete P; return fail(MOMENT_EINVAL, "moment_plan: hbm_cap must be positive"); }
    P->t_nvlink = max_link == 0 ? 0 : ceil_div((u128)max_link, (u128)a->nvlink_cap);
    P->t_hbm = ceil_div((u128)max_hbm, (u128)a->hbm_cap);
    P->t_star = std::max(P->t_ingest, std::max(P->t_nvlink, P->t_hbm));
    *out = P;
    return MOMENT_OK;
}

extern "C" moment_status moment_replicate_search(moment_topo_t T, const moment_replicate_args* a, int64_t* t_star,
                                                int32_t* best) {
    if (!T || !a || !a->place || !t_star || !best || (a->n_candidates > 0 && !a->candidates))
        return fail(MOMENT_EINVAL, "moment_replicate_search: null argument");
    const moment_place_args* pa = a->place;
    const int64_t n = pa->n_vertices;
    if (pa->mode != MOMENT_PLACE_DDAK) return fail(MOMENT_EINVAL, "moment_replicate_search: place mode must be DDAK");
    if (n < 0 || n >= (int64_t(1) << 32)) return fail(MOMENT_EINVAL, "moment_replicate_search: n_vertices out of range");
    if (n > 0 && !pa->hotness) return fail(MOMENT_EINVAL, "moment_replicate_search: hotness is null");
    if (a->row_bytes <= 0 || a->hot_batches <= 0 || a->n_candidates < 0 || (a->demand_counts && a->demand_batches <= 0))
        return fail(MOMENT_EINVAL, "moment_replicate_search: row_bytes, hot_batches, demand_batches must be > 0");
    const uint64_t* dem = a->demand_counts ? a->demand_counts : pa->hotness;
    const int64_t dem_batches = a->demand_counts ? a->demand_batches : a->hot_batches;
    std::vector<Bin> bins0;
    std::vector<int32_t> bin_node;
    MOMENT_TRY(resolve_bins(T, pa, bins0, bin_node));
    const int N = (int)T->nodes.size();
    for (size_t b = 0; b < bin_node.size(); b++)
        if (bin_node[b] < 0 || bin_node[b] >= N || T->nodes[bin_node[b]].kind != MOMENT_NODE_STORAGE)
            return fail(MOMENT_EINVAL, "moment_replicate_search: bin %zu is not a storage node", b);
    std::vector<uint32_t> order;
    order_by_hotness(n, pa->hotness, order);
    const int64_t pool = pa->pool > 0 ? pa->pool : 100;
    *best = -1;
    auto demand = [&](uint64_t acc) -> int64_t {
        return (int64_t)(((u128)acc * (u128)(uint64_t)a->row_bytes) / (u128)(uint64_t)dem_batches);
    };
    for (int32_t i = 0; i < a->n_candidates; i++) {
        t_star[i] = -1;
        if (a->candidates[i] < 0) return fail(MOMENT_EINVAL, "moment_replicate_search: candidate %d is negative", i);
        if (a->candidates[i] > n) continue;  // more replicas than vertices: infeasible
        std::vector<Bin> bins = bins0;
        uint64_t rep = 0;
        moment_status st = ddak_core(n, pa->hotness, order, a->candidates[i], pool, bins, nullptr, nullptr, nullptr,
                                     dem, &rep);
        if (st == MOMENT_EINFEASIBLE) continue;
        if (st != MOMENT_OK) return st;
        std::vector<int64_t> d(N, 0);
        for (size_t b = 0; b < bins.size(); b++) d[bin_node[b]] += demand(bins[b].demand);
        moment_plan_args pl{};
        pl.k = a->k;
        pl.gpu_node = a->gpu_node;
        pl.bin_demand_bytes = d.data();
        pl.nvlink_cap = a->nvlink_cap;
        pl.hbm_cap = a->hbm_cap;
        pl.replica_demand_bytes = demand(rep);
        moment_plan_t P = nullptr;
        st = moment_plan(T, &pl, &P);
        if (st == MOMENT_EINFEASIBLE) continue;
        if (st != MOMENT_OK) return st;
        t_star[i] = P->t_star;
        moment_plan_free(P);
        if (*best < 0 || t_star[i] < t_star[*best]) *best = i;
    }
    return MOMENT_OK;
}

extern "C" moment_status moment_plan_info(moment_plan_t P, int64_t* t_star, int64_t* t_ingest, int64_t* t_nvlink,
                                          int64_t* t_hbm, int64_t* link_flow, int64_t* quota) {
    if (!P) return fail(MOMENT_EINVAL, "moment_plan_info: null plan");
    if (t_star) *t_star = P->t_star;
    if (t_ingest) *t_ingest = P->t_ingest;
    if (t_nvlink) *t_nvlink = P->t_nvlink;
    if (t_hbm) *t_hbm = P->t_hbm;
    if (link_flow) std::memcpy(link_flow, P->link_flow.data(), P->link_flow.size() * sizeof(int64_t));
    if (quota) std::memcpy(quota, P->quota.data(), P->quota.size() * sizeof(int64_t));
    return MOMENT_OK;
}

extern "C" moment_status moment_plan_free(moment_plan_t P) {
    delete P;
    return MOMENT_OK;
}

extern "C" const char* moment_last_error(void) { return moment::last_error(); }
extern "C" int32_t moment_version(void) { return (0 << 16) | 2; }
