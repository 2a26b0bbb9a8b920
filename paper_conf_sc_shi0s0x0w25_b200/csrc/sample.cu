// sample.cu — H1-H3: multi-hop neighbour sampling with dedup/relabel on sm_100a (R3-R6).
//
// One sample call is 2H + 1 kernels (2H + 2 with a separate init) and no memsets. No kernel needs the host
// to know |F_h| or E_h (every size is read from device memory), so the call is CUDA-graph capturable. The
// critical path per hop is two kernels; offsets, compaction and relabelling of every hop happen once:
//   init        : F_0 = seeds; lidx / visited of the seeds; zero the tile descriptors and tickets (done by
//                 the first hop's sampler, or a separate kernel).
//   sample (h)  : one k-lane group per frontier node v draws min(deg v, k) Floyd (or with-replacement)
//                 positions from Philox (choices resolved in parallel), writes the neighbour ids to the
//                 node's k-slot row of a padded buffer, its count to cnt_h, adds it to its compaction
//                 tile's edge sum, and marks the ids in `newbits`.
//   bitscan (h) : F_{h+1} = F_h ++ (newbits & ~visited) in ascending id order: chained scan of bitmap
//                 popcounts (1024 words per tile) gives each new id its position. Sparse scan (large graphs):
//                 lidx[id] = position. Dense scan (rank relabelling): no lidx write; instead rel_h[w] = {new
//                 bits of word w, rank of its first new id} for every word (a sequential, L2-resident table).
//   compact     : every tile's global edge position from the per-tile edge sums (no chaining) -> per-hop
//                 offsets, E_h, and src = position of the padded id (lidx[id], or from rel: the latest hop
//                 hh <= h whose word has the id's bit, counts[hh] + rank + popc of the lower bits; seeds via
//                 lidx) copied into the packed output; then clears `visited` for F_H.
#include <cooperative_groups.h>

#include <algorithm>
#include <climits>
#include <cstdlib>

#include "ctx.h"
#include "device_util.cuh"

namespace cg = cooperative_groups;

namespace moment {
namespace {

constexpr int kScanWords = kBitscanWordsPerThread;  // bitmap words per bitscan thread (uint4 loads)
constexpr int kScanTileWords = kBitscanTileWords;   // words per tile
static_assert(kScanWords % 4 == 0, "bitscan loads whole uint4s");
constexpr int kMaxHops = 16;
#ifndef MOMENT_SAMPLE_MIN_BLOCKS
#define MOMENT_SAMPLE_MIN_BLOCKS 8  // __launch_bounds__ min blocks per SM of the sampler kernels (<= 32 registers,
                                    // the SM's full 2048 threads: round 2, one node per group, +1.5 % per step vs 6 /
                                    // 40 registers, which measured +5-8 % over uncapped in round 1)
#endif

struct HopArgs {
    const int64_t* indptr;
    const int32_t* indices;
    const int64_t* nodes;
    const int64_t* counts;
    int32_t* pad;      // [F_bound_h * k]: node idx's samples at pad[idx * k + r]
    int32_t* cnt;      // [F_bound_h]: samples of node idx
    uint32_t* newbits;
    uint32_t* summary;     // sparse scan only (else null): bit w of summary = newbits word w was marked
    const uint64_t* call;  // device call block: [0] = rng_seed, [1] = seeds pointer (written per call)
    int32_t h, k;
    int32_t replace;
    int32_t grid_per_sm;   // launch cap: blocks per SM (grid-stride beyond it)
    // this hop's edges per compaction tile (kSampleTile consecutive nodes), summed here so that the
    // compaction needs no chained scan; zeroed before the hop (hop 0: set_call, hop h: bitscan h - 1)
    unsigned long long* tile_edges;
    // 1: every sampled id's indptr line is prefetched into L2 (evict_last) for the next hop (MOMENT_HOP_PREFETCH;
    // not on the last hop); 2: the same without the eviction hint
    int32_t prefetch_next;
};

// The per-call initialisation that the first hop's sampler does itself (hop_sample_warp_kernel<Q, true>):
// F_0 = seeds (read from the call block), their lidx / visited entries, the seed checks, and zeroed tile
// descriptors, tickets and hop bases for the scans that follow.
struct InitArgs {
    int64_t n_seeds, n_vertices;
    int64_t* nodes;
    int64_t* counts;
    int32_t* lidx;
    uint32_t* visited;
    uint32_t* error_flag;
    int32_t check;
    uint64_t* tile_status;
    int64_t n_tile_status;
    uint32_t* tickets;
    int32_t n_tickets;
    uint64_t* ebase;
    int32_t n_ebase;
};

// Fire-and-forget: the result is unused, so this is a RED.OR the issuing warp never waits on.
// Sparse scan (large graphs): the newbits word's bit in `summary` is marked too, so that the bitscan reads
// only the words a hop touched instead of the whole n-bit bitmap.
__device__ __forceinline__ void mark_new(const HopArgs& a, int32_t u) {
    atomicOr(a.newbits + (u >> 5), 1u << (u & 31));
    if (a.summary) atomicOr(a.summary + (u >> 10), 1u << ((u >> 5) & 31));
    if (a.prefetch_next == 1) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(a.indptr + u));
    else if (a.prefetch_next == 2) asm volatile("prefetch.global.L2 [%0];" ::"l"(a.indptr + u));
}

// Floyd's k choices for node v at hop h, lane i < k owning choice i (k <= G): t_i = uniform(draw(i),
// j_i + 1), j_i = d - k + i, and c_i = j_i if t_i is already in S_{i-1} = {c_0..c_{i-1}}, else t_i.
// Resolved without the k-step sequential chain: t_i is in S_{i-1} iff (a) some earlier t_l equals t_i
// (if t_l was itself a duplicate it was already in S) or (b) t_i = j_l for an earlier l whose choice was
// j_l. (a) is one match_any; (b) refers only to earlier lanes, so a fixpoint over ballots converges.
template <int G>
__device__ __forceinline__ int32_t floyd_choice(const cg::thread_block_tile<G>& grp, uint64_t seed, int64_t v, int h,
                                                int32_t d, int k) {
    const int lane = grp.thread_rank();
    const bool active = lane < k;
    const int32_t jj = d - k + lane;
    const int32_t t = active ? (int32_t)dev::uniform(dev::draw(seed, v, h, lane), (uint32_t)(jj + 1)) : -1 - lane;
    const unsigned below = (1u << lane) - 1u;
    const unsigned same = grp.match_any(t);
    const bool dup_a = active && (same & below) != 0;
    const int lstar = t - (d - k);  // the earlier lane whose j equals t, if any
    const bool ref = active && !dup_a && t >= d - k && lstar < lane;
    unsigned dup = grp.ballot(dup_a);
    for (;;) {
        const bool now = dup_a || (ref && ((dup >> lstar) & 1u));
        const unsigned nd = grp.ballot(now);
        if (nd == dup) break;
        dup = nd;
    }
    return ((dup >> lane) & 1u) ? jj : t;
}

// Positions for k > 32 (G == 32): chunks of 32 choices resolved in draw order; earlier chunks are final
// and kept (as positions) in `out`, then sorted and replaced by ids. Rare (fanout > 32).
__device__ void sample_node_wide(const cg::thread_block_tile<32>& grp, const HopArgs& a, uint64_t seed, int64_t v,
                                 int64_t lo, int32_t d, int32_t* out) {
    const int lane = grp.thread_rank();
    const int k = a.k;
    for (int c0 = 0; c0 < k; c0 += 32) {
        const int i = c0 + lane;
        int32_t j = 0, t = 0, c = -1;
        bool prev_hit = false;
        if (i < k) {
            j = d - k + i;
            t = (int32_t)dev::uniform(dev::draw(seed, v, a.h, i), (uint32_t)(j + 1));
            for (int q = 0; q < c0; q++) prev_hit |= out[q] == t;
        }
        const int nm = min(32, k - c0);
        for (int m = 0; m < nm; m++) {
            const int32_t tm = grp.shfl(t, m);
            const unsigned any = grp.ballot(lane < m && c == tm);
            if (lane == m) c = (any || prev_hit) ? j : t;
        }
        grp.sync();
        if (i < k) out[i] = c;
        grp.sync();
    }
    int32_t mine[kMaxFanout / 32];
    int rk[kMaxFanout / 32];
    const int per = (k + 31) / 32;
    for (int q = 0; q < per; q++) {
        const int i = q * 32 + lane;
        mine[q] = i < k ? out[i] : 0;
        int r = 0;
        if (i < k)
            for (int l = 0; l < k; l++) r += out[l] < mine[q];
        rk[q] = r;
    }
    grp.sync();
    for (int q = 0; q < per; q++) {
        const int i = q * 32 + lane;
        if (i < k) {
            const int32_t u = __ldg(a.indices + lo + mine[q]);
            out[rk[q]] = u;
            mark_new(a, u);
        }
    }
}

// Nodes with fanout > G (G == 32 only, fanout > 32): per-node paths without the register batching.
template <int G>
__device__ __forceinline__ void sample_node_slow(const cg::thread_block_tile<G>& grp, const HopArgs& a, uint64_t seed,
                                                 int64_t v, int64_t lo, int32_t d, int32_t* out) {
    const int lane = grp.thread_rank();
    const int k = a.k;
    if (a.replace) {
        for (int i = lane; i < k; i += G) {
            const int32_t u = __ldg(a.indices + lo + dev::uniform(dev::draw(seed, v, a.h, i), (uint32_t)d));
            out[i] = u;
            mark_new(a, u);
        }
    } else if (d <= k) {
        for (int p = lane; p < d; p += G) {
            const int32_t u = __ldg(a.indices + lo + p);
            out[p] = u;
            mark_new(a, u);
        }
    } else {
        if constexpr (G == 32) sample_node_wide(grp, a, seed, v, lo, d, out);
    }
}

// One G-lane group handles Q consecutive frontier nodes per step (grid-stride): their node ids, degrees,
// choices (lane i owns choice i: Floyd / all / with replacement) and neighbour loads are issued as Q
// independent batches, so each thread keeps Q dependent chains in flight instead of one.
template <int G, int Q>
__global__ void __launch_bounds__(256, MOMENT_SAMPLE_MIN_BLOCKS) hop_sample_kernel(HopArgs a) {
    const int64_t F = a.counts[a.h];
    const uint64_t seed = a.call[0];
    auto grp = cg::tiled_partition<G>(cg::this_thread_block());
    const int lane = grp.thread_rank();
    const int k = a.k;
    const int64_t groups = (int64_t)gridDim.x * (256 / G);
    for (int64_t base = ((int64_t)blockIdx.x * (256 / G) + threadIdx.x / G) * Q; base < F; base += groups * Q) {
        int64_t v[Q], lo[Q];
        int32_t d[Q], pos[Q], rnk[Q], u[Q];
#pragma unroll
        for (int q = 0; q < Q; q++) v[q] = base + q < F ? a.nodes[base + q] : -1;
#pragma unroll
        for (int q = 0; q < Q; q++) {
            lo[q] = 0;
            d[q] = 0;
            if (v[q] >= 0) {
                lo[q] = dev::ld_rand(a.indptr + v[q]);
                d[q] = (int32_t)(dev::ld_rand(a.indptr + v[q] + 1) - lo[q]);
            }
        }
#pragma unroll
        for (int q = 0; q < Q; q++) {
            pos[q] = -1;
            rnk[q] = 0;
            const int32_t dq = d[q];
            if (dq <= 0 || k > G) continue;  // uniform per group
            if (a.replace) {
                if (lane < k) {
                    pos[q] = (int32_t)dev::uniform(dev::draw(seed, v[q], a.h, lane), (uint32_t)dq);
                    rnk[q] = lane;
                }
            } else if (dq <= k) {
                if (lane < dq) {
                    pos[q] = lane;
                    rnk[q] = lane;
                }
            } else {
                const int32_t ch = floyd_choice<G>(grp, seed, v[q], a.h, dq, k);
                int r = 0;
#pragma unroll
                for (int l = 0; l < G; l++) {
                    const int32_t cl = grp.shfl(ch, l);
                    r += (l < k) && cl < ch;
                }
                if (lane < k) {
                    pos[q] = ch;
                    rnk[q] = r;
                }
            }
        }
#pragma unroll
        for (int q = 0; q < Q; q++) u[q] = pos[q] >= 0 ? dev::ld_rand(a.indices + lo[q] + pos[q]) : 0;
#pragma unroll
        for (int q = 0; q < Q; q++) {
            const int64_t idx = base + q;
            if (idx >= F) break;
            if (lane == 0) {
                const int32_t c = a.replace ? (d[q] > 0 ? k : 0) : min(d[q], k);
                a.cnt[idx] = c;
                if (c) atomicAdd(a.tile_edges + idx / kSampleTile, (unsigned long long)c);
            }
            if (pos[q] >= 0) {
                a.pad[idx * k + rnk[q]] = u[q];
                mark_new(a, u[q]);
            }
        }
        if (k > G) {
            for (int q = 0; q < Q; q++) {
                const int64_t idx = base + q;
                if (idx >= F) break;
                if (d[q] > 0) sample_node_slow<G>(grp, a, seed, v[q], lo[q], d[q], a.pad + idx * k);
            }
        }
    }
}

// Warp-segmented sampler for k <= 32: a warp holds NG = floor(32 / k) groups of exactly k lanes (lane i of
// group g owns choice i), so 32 mod k lanes idle instead of G - k per power-of-two tile (k = 5: 30 of 32
// lanes busy, not 20). Control flow is warp-uniform: every group runs the same steps under per-group
// predicates and the collectives span the whole warp (match_any keyed by (group, t), ballots read at the
// group's bit offset), so groups never diverge and no convergence barriers are needed. Step q of a warp
// handles the NG consecutive frontier nodes base + q * NG + g: its pad stores are one run of NG * k ints.
// Same choices as floyd_choice (same draws, same resolution rule), only the lane layout differs.
template <int Q, bool kInit>
__global__ void __launch_bounds__(256, MOMENT_SAMPLE_MIN_BLOCKS) hop_sample_warp_kernel(HopArgs a, InitArgs in) {
    constexpr unsigned kFull = 0xffffffffu;
    const int64_t F = kInit ? in.n_seeds : a.counts[a.h];
    const uint64_t seed = a.call[0];
    const int64_t* seeds = kInit ? reinterpret_cast<const int64_t*>(a.call[1]) : nullptr;
    if (kInit) {
        const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (int64_t)gridDim.x * blockDim.x;
        for (int64_t j = tid; j < in.n_tile_status; j += nth) in.tile_status[j] = 0;
        for (int64_t j = tid; j < in.n_tickets; j += nth) in.tickets[j] = 0;
        for (int64_t j = tid; j < in.n_ebase; j += nth) in.ebase[j] = 0;
        if (tid == 0) in.counts[0] = in.n_seeds;
    }
    const int k = a.k;
    const int lane = threadIdx.x & 31;
    const int NG = 32 / k;
    const int g = lane / k;  // NG for the idle lanes
    const int i = lane - g * k;
    const bool live = g < NG;
    const int gbase = g * k;
    const unsigned below = (1u << lane) - 1u;
    // lanes of this lane's group (a 32-bit match keyed by t alone, masked to the group, replaces a 64-bit
    // match keyed by (group, t)); idle lanes never take part in a Floyd resolution
    const unsigned gmask = (k >= 32 ? kFull : (1u << k) - 1u) << gbase;
    // ranks of the chosen positions: every group's k choices go through shared memory (a slot of ks >= k
    // ints per group, padded with INT_MAX) and each lane counts the smaller ones with 16-byte loads,
    // ceil(k / 4) loads instead of k shuffles
    __shared__ __align__(16) int32_t s_rank[8][128];
    int32_t* const sw = s_rank[threadIdx.x >> 5];
    const int ks = (k + 3) & ~3;
    const int64_t per_warp = (int64_t)NG * Q;
    const int64_t warps = (int64_t)gridDim.x * 8;
    for (int64_t base = ((int64_t)blockIdx.x * 8 + threadIdx.x / 32) * per_warp; base < F; base += warps * per_warp) {
        int64_t idx[Q], v[Q], lo[Q];
        int32_t d[Q], pos[Q], rnk[Q], u[Q];
#pragma unroll
        for (int q = 0; q < Q; q++) {
            idx[q] = base + (int64_t)q * NG + g;
            if (kInit) {  // F_0 = seeds; an out-of-range seed is flagged and replaced by vertex 0 (never written)
                v[q] = -1;
                if (live && idx[q] < F) {
                    const int64_t sv = seeds[idx[q]];
                    const bool bad = sv < 0 || sv >= in.n_vertices;
                    v[q] = bad ? 0 : sv;
                    if (i == 0) {
                        in.nodes[idx[q]] = v[q];
                        if (bad) {
                            atomicOr(in.error_flag, 1u);
                        } else {
                            in.lidx[sv] = (int32_t)idx[q];
                            const uint32_t bit = 1u << (sv & 31);
                            const uint32_t old = atomicOr(in.visited + (sv >> 5), bit);
                            if (in.check && (old & bit)) atomicOr(in.error_flag, 2u);
                        }
                    }
                }
            } else {
                v[q] = (live && idx[q] < F) ? a.nodes[idx[q]] : -1;
            }
        }
#pragma unroll
        for (int q = 0; q < Q; q++) {
            lo[q] = 0;
            d[q] = 0;
            if (v[q] >= 0) {
                lo[q] = dev::ld_rand(a.indptr + v[q]);
                d[q] = (int32_t)(dev::ld_rand(a.indptr + v[q] + 1) - lo[q]);
            }
        }
#pragma unroll
        for (int q = 0; q < Q; q++) {
            const int32_t dq = d[q];
            pos[q] = -1;
            rnk[q] = i;
            if (a.replace) {  // uniform over the launch
                if (dq > 0) pos[q] = (int32_t)dev::uniform(dev::draw(seed, v[q], a.h, i), (uint32_t)dq);
                continue;
            }
            const bool floyd = dq > k;
            if (!floyd && i < dq) pos[q] = i;  // d <= k: every neighbour, in CSR order
            if (!__any_sync(kFull, floyd)) continue;
            const int32_t jj = dq - k + i;
            const int32_t t = floyd ? (int32_t)dev::uniform(dev::draw(seed, v[q], a.h, i), (uint32_t)(jj + 1))
                                    : -1 - lane;  // unique sentinel: never matches
            const unsigned same = __match_any_sync(kFull, (uint32_t)t) & gmask;
            const bool dup_a = floyd && (same & below) != 0;
            const int lstar = gbase + (t - (dq - k));  // the earlier lane of this group whose j equals t
            const bool ref = floyd && !dup_a && t >= dq - k && lstar < lane;
            unsigned dup = __ballot_sync(kFull, dup_a);
            for (;;) {
                const bool now = dup_a || (ref && ((dup >> lstar) & 1u));
                const unsigned nd = __ballot_sync(kFull, now);
                if (nd == dup) break;
                dup = nd;
            }
            const int32_t c = ((dup >> lane) & 1u) ? jj : t;
            int r = 0;
            if (k > 1) {
                if (live) {
                    sw[g * ks + i] = c;
                    for (int p = k + i; p < ks; p += k) sw[g * ks + p] = INT_MAX;
                }
                __syncwarp();
                if (live) {
                    const int4* row = reinterpret_cast<const int4*>(sw + g * ks);
                    for (int l4 = 0; l4 < ks / 4; l4++) {
                        const int4 x = row[l4];
                        r += (x.x < c) + (x.y < c) + (x.z < c) + (x.w < c);
                    }
                }
                __syncwarp();  // the slots are rewritten by the next node step
            }
            if (floyd) {
                pos[q] = c;
                rnk[q] = r;
            }
        }
#pragma unroll
        for (int q = 0; q < Q; q++) u[q] = pos[q] >= 0 ? dev::ld_rand(a.indices + lo[q] + pos[q]) : 0;
        // the warp's step covers nodes [base, base + NG * Q) (<= 128 < kSampleTile), so at most two
        // compaction tiles: tile_a and the one after it; one warp reduction and RED per tile and step
        const int64_t tile_a = base / kSampleTile, bound = (tile_a + 1) * kSampleTile;
        uint32_t sum_a = 0, sum_b = 0;
#pragma unroll
        for (int q = 0; q < Q; q++) {
            const bool node = live && idx[q] < F;
            const uint32_t c = node ? (uint32_t)(a.replace ? (d[q] > 0 ? k : 0) : min(d[q], k)) : 0u;
            if (node && i == 0) {
                a.cnt[idx[q]] = (int32_t)c;
                if (idx[q] < bound) sum_a += c;
                else sum_b += c;
            }
            if (node && pos[q] >= 0) {
                a.pad[idx[q] * k + rnk[q]] = u[q];
                mark_new(a, u[q]);
            }
        }
        sum_a = __reduce_add_sync(kFull, sum_a);
        sum_b = __reduce_add_sync(kFull, sum_b);
        if (lane == 0) {
            if (sum_a) atomicAdd(a.tile_edges + tile_a, (unsigned long long)sum_a);
            if (sum_b) atomicAdd(a.tile_edges + tile_a + 1, (unsigned long long)sum_b);
        }
    }
}

// the bitscan's neighbour-list prefetch pays only while the CSR is L2-sized: C1 (1 M edges, 4 MB of indices)
// 98.7 -> 109 M seeds/s, C2 (62 M edges) 36.7 -> 35.6 (profiles/r01_hop_prefetch.txt)
constexpr int64_t kScanPrefetchMaxEdges = int64_t(8) << 20;

struct ScanArgs {
    int64_t* nodes;
    int64_t* counts;
    int32_t* lidx;
    uint32_t* newbits;
    uint32_t* visited;
    uint32_t* summary;  // sparse scan: touched-word bitmap of newbits (cleared here)
    uint64_t* tile_status;
    uint32_t* ticket;
    int64_t n_words;
    int32_t h;
    unsigned long long* zero;  // the next hop's compaction tile sums, zeroed here (before that hop runs)
    int64_t n_zero;
    // dense scan with rank relabelling (else null): rel[w] = {new-id bits of word w at this hop, rank of the
    // word's first new id among the hop's new ids}, written for EVERY word (no clearing needed); lidx is then
    // not written for non-seed ids and the compaction finds an id's position from rel (L2-resident)
    uint2* rel;
    // sparse scan with rank relabelling (else null): per summary word sw, srel[sw] = {mask of its newbits
    // words that hold new ids, index of its first entry in trel}; trel[e] = {new-id bits, rank of the word's
    // first new id} for the words with new ids, in id order (a second count, packed into the scan's value)
    uint2* srel;
    uint2* trel;
    // dense scan, not the last hop (else 0): each new id's CSR row start is read (its indptr line is already
    // L2-resident from the sampler's prefetch) and the first line of its neighbour list is prefetched into L2
    // (evict_last) for the next hop's sampler (MOMENT_SCAN_PREFETCH)
    const int64_t* indptr;
    const int32_t* indices;
    int32_t prefetch_idx;
};

// F_{h+1} = F_h ++ ascending ids set in (newbits & ~visited).
// kPrefetch: a separate instantiation, so the default scan's code is not touched by the prefetch branch (the
// runtime-flag version slowed the C2 scans by ~20 % with the flag off)
// Register caps (round 2): with 16+ batches in flight the SMs' register files decide how many of the lanes'
// kernels are resident at once, so the dense bitscan is held to 40 registers (3 x 512-thread blocks per SM;
// uncapped it took 80) and the compaction to 40 (6 x 256-thread blocks per SM, 6 slots in flight; was 64 with
// 8): sampling-only 13.3 -> 11.5 us per batch at 16 lanes, the full step -1 %, the driver's K = 20 +2 %
// (tools/ab_multi.sh, profiles/r02_sampler_experiments.txt)
#ifndef MOMENT_SCAN_MINB
#define MOMENT_SCAN_MINB 3
#endif
template <bool kPrefetch>
__global__ void __launch_bounds__(kBitscanThreads, MOMENT_SCAN_MINB) bitscan_kernel(ScanArgs a) {
    __shared__ int64_t s_red[kBitscanThreads / 32];
    __shared__ uint32_t s_tile;
    __shared__ int s_nearest;
    const int64_t F = a.counts[a.h];
    const int64_t n_tiles = (a.n_words + kScanTileWords - 1) / kScanTileWords;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < a.n_zero; j += (int64_t)gridDim.x * blockDim.x)
        a.zero[j] = 0;
    for (;;) {
        if (threadIdx.x == 0) s_tile = atomicAdd(a.ticket, 1u);
        __syncthreads();
        const int64_t tile = s_tile;
        if (tile >= n_tiles) break;
        const int64_t w0 = tile * kScanTileWords + (int64_t)threadIdx.x * kScanWords;
        uint32_t nb[kScanWords], vs[kScanWords];
        if (w0 + kScanWords <= a.n_words) {
#pragma unroll
            for (int q4 = 0; q4 < kScanWords / 4; q4++) {
                const uint4 n4 = __ldcg(reinterpret_cast<const uint4*>(a.newbits + w0) + q4);
                const uint4 v4 = __ldcg(reinterpret_cast<const uint4*>(a.visited + w0) + q4);
                nb[4 * q4] = n4.x; nb[4 * q4 + 1] = n4.y; nb[4 * q4 + 2] = n4.z; nb[4 * q4 + 3] = n4.w;
                vs[4 * q4] = v4.x; vs[4 * q4 + 1] = v4.y; vs[4 * q4 + 2] = v4.z; vs[4 * q4 + 3] = v4.w;
            }
        } else {
#pragma unroll
            for (int q = 0; q < kScanWords; q++) {
                const int64_t w = w0 + q;
                nb[q] = w < a.n_words ? __ldcg(a.newbits + w) : 0u;
                vs[q] = w < a.n_words ? __ldcg(a.visited + w) : 0u;
            }
        }
        int cnt = 0;
#pragma unroll
        for (int q = 0; q < kScanWords; q++) cnt += __popc(nb[q] & ~vs[q]);
        int64_t agg;
        const int64_t excl = dev::block_exclusive_scan<kBitscanThreads>(cnt, &agg, s_red);
        const int64_t prefix = dev::lookback_block<kBitscanThreads>(a.tile_status, tile, agg, s_red, &s_nearest);
        int64_t pos = F + prefix + excl;
        if (tile == n_tiles - 1 && threadIdx.x == 0) a.counts[a.h + 1] = F + prefix + agg;
        uint32_t rk[kScanWords];
#pragma unroll
        for (int q = 0; q < kScanWords; q++) {
            const int64_t w = w0 + q;
            const uint32_t nw = nb[q] & ~vs[q];
            rk[q] = (uint32_t)(pos - F);
            uint32_t bits = nw;
            while (bits) {
                const int b = __ffs(bits) - 1;
                bits &= bits - 1;
                const int64_t id = w * 32 + b;
                a.nodes[pos] = id;
                if (!a.rel) a.lidx[id] = (int32_t)pos;
                if (kPrefetch)
                    asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(a.indices + __ldcg(a.indptr + id)));
                pos++;
            }
            if (nb[q]) a.newbits[w] = 0u;
            if (nw) a.visited[w] = vs[q] | nw;  // no re-read: the tile owns its words
        }
        if (a.rel) {  // rel is padded to whole tiles: every thread's words exist
            uint4* r4 = reinterpret_cast<uint4*>(a.rel + w0);
#pragma unroll
            for (int q = 0; q < kScanWords; q += 2)
                r4[q / 2] = make_uint4(nb[q] & ~vs[q], rk[q], nb[q + 1] & ~vs[q + 1], rk[q + 1]);
        }
        __syncthreads();
    }
}

// Sparse variant for large graphs (n_words >> touched words): a tile is kSparseTileWords newbits words =
// one summary word per thread; a thread reads only the newbits / visited words whose summary bit is set
// (the words the hop marked), 4 at a time, so the scan costs O(touched words + n / 1024) instead of
// O(n / 32). Same result and order as bitscan_kernel: a thread's words are consecutive and its ids
// ascending, threads of a tile and tiles are in id order.

template <typename Fn>
__device__ __forceinline__ void for_touched_words(uint32_t sm, const uint32_t* newbits, const uint32_t* visited,
                                                  int64_t w_base, Fn fn) {
    while (sm) {
        int wi[4];
        uint32_t nb[4], vs[4];
#pragma unroll
        for (int j = 0; j < 4; j++) {
            wi[j] = sm ? __ffs(sm) - 1 : -1;
            sm &= sm - 1;
        }
#pragma unroll
        for (int j = 0; j < 4; j++) {
            nb[j] = wi[j] >= 0 ? __ldcg(newbits + w_base + wi[j]) : 0u;
            vs[j] = wi[j] >= 0 ? __ldcg(visited + w_base + wi[j]) : 0u;
        }
#pragma unroll
        for (int j = 0; j < 4; j++)
            if (wi[j] >= 0) fn(w_base + wi[j], nb[j], vs[j]);
    }
}

template <int NT>
__global__ void __launch_bounds__(NT) bitscan_sparse_kernel(ScanArgs a) {
    constexpr int kSparseTileWords = 32 * NT;
    __shared__ int64_t s_red[NT / 32];
    __shared__ uint32_t s_tile;
    __shared__ int s_nearest;
    const int64_t F = a.counts[a.h];
    const int64_t n_tiles = (a.n_words + kSparseTileWords - 1) / kSparseTileWords;
    const int64_t n_summary = (a.n_words + 31) / 32;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < a.n_zero; j += (int64_t)gridDim.x * blockDim.x)
        a.zero[j] = 0;
    for (;;) {
        if (threadIdx.x == 0) s_tile = atomicAdd(a.ticket, 1u);
        __syncthreads();
        const int64_t tile = s_tile;
        if (tile >= n_tiles) break;
        const int64_t sw = tile * NT + threadIdx.x;  // this thread's summary word
        const uint32_t sm = sw < n_summary ? __ldcg(a.summary + sw) : 0u;
        const int64_t w_base = sw * 32;
        // scanned value: new ids in the low 32 bits; with rank relabelling also the words holding new ids
        // (trel entries) in the high bits — one scan and look-back serve both prefixes
        int64_t val = 0;
        uint32_t emask = 0;  // words of this summary word that hold new ids
        for_touched_words(sm, a.newbits, a.visited, w_base, [&](int64_t w, uint32_t nb, uint32_t vs) {
            const uint32_t nw = nb & ~vs;
            val += __popc(nw);
            if (nw) emask |= 1u << (uint32_t)(w - w_base);
        });
        if (a.srel) val += (int64_t)__popc(emask) << 32;
        int64_t agg;
        const int64_t excl = dev::block_exclusive_scan<NT>(val, &agg, s_red);
        const int64_t prefix = dev::lookback_block<NT>(a.tile_status, tile, agg, s_red, &s_nearest);
        const int64_t before = prefix + excl;
        int64_t pos = F + (before & 0xFFFFFFFFll);
        int64_t ent = before >> 32;
        if (tile == n_tiles - 1 && threadIdx.x == 0) a.counts[a.h + 1] = F + ((prefix + agg) & 0xFFFFFFFFll);
        if (a.srel && sw < n_summary) a.srel[sw] = make_uint2(emask, (uint32_t)ent);
        for_touched_words(sm, a.newbits, a.visited, w_base, [&](int64_t w, uint32_t nb, uint32_t vs) {
            const uint32_t nw = nb & ~vs;
            if (a.srel && nw) a.trel[ent++] = make_uint2(nw, (uint32_t)(pos - F));
            uint32_t bits = nw;
            while (bits) {
                const int b = __ffs(bits) - 1;
                bits &= bits - 1;
                const int64_t id = w * 32 + b;
                a.nodes[pos] = id;
                if (!a.srel) a.lidx[id] = (int32_t)pos;
                pos++;
            }
            a.newbits[w] = 0u;
            if (nw) a.visited[w] = vs | nw;
        });
        if (sm) a.summary[sw] = 0u;
        __syncthreads();
    }
}

struct CompactArgs {
    int64_t* offsets;
    int32_t* src;
    int64_t* counts;
    const int64_t* nodes;
    const int32_t* lidx;
    uint32_t* visited;
    const unsigned long long* tile_edges;  // edges per tile, tiles of all hops numbered by the bounds tb[]
    int32_t H;
    int64_t tb[kMaxHops + 1];  // first tile of hop h (sum of ceil(F_bound_h' / kSampleTile), h' < h)
    int32_t k[kMaxHops];
    uint32_t kmagic[kMaxHops];  // ceil(2^32 / k): slot / k = umulhi(slot, kmagic) for slot < 2^18, k <= 1024
    const int32_t* pad[kMaxHops];
    const int32_t* cnt[kMaxHops];
    const uint2* rel;    // dense scan with rank relabelling: hop h's rel at rel + h * rel_stride, else null
    int64_t rel_stride;
    const uint2* srel;   // sparse scan with rank relabelling: hop h's tables at srel + h * srel_stride and
    const uint2* trel[kMaxHops];  //   trel[h], else null
    int64_t srel_stride;
    const uint64_t* call;  // the call block: [2] = mapped host counts of moment_step_host, or 0
    uint32_t* done;        // blocks finished (zeroed per call with the tickets)
};

// Sparse scan's two-level tables: is v new at hop hh, and at which position?
__device__ __forceinline__ bool srel_probe(const CompactArgs& a, int32_t v, int hh, int32_t* out) {
    const uint32_t w = (uint32_t)v >> 5, j = w & 31;
    const uint2 m = __ldcg(a.srel + hh * a.srel_stride + (w >> 5));
    if (!((m.x >> j) & 1u)) return false;
    const uint2 r = __ldcg(a.trel[hh] + m.y + __popc(m.x & ((1u << j) - 1u)));
    const uint32_t bit = 1u << (v & 31);
    if (!(r.x & bit)) return false;
    *out = (int32_t)(a.counts[hh] + r.y + __popc(r.x & (bit - 1)));
    return true;
}

// Position in F_{h+1} of an id sampled at hop h, from the bitscans' rel tables (rank relabelling): the id
// is new at the latest hop hh <= h whose rel word has its bit, at counts[hh] + the word's rank + the bits
// below it in the word; an id in no table is a seed, whose position lidx holds.
__device__ __forceinline__ int32_t rel_position(const CompactArgs& a, int32_t v, int hh) {
    const uint32_t bit = 1u << (v & 31);
    if (a.srel) {
        int32_t p;
        for (; hh >= 0; hh--)
            if (srel_probe(a, v, hh, &p)) return p;
        return dev::ld_rand(a.lidx + v);
    }
    for (; hh >= 0; hh--) {
        const uint2 r = __ldcg(a.rel + hh * a.rel_stride + (v >> 5));
        if (r.x & bit) return (int32_t)(a.counts[hh] + r.y + __popc(r.x & (bit - 1)));
    }
    return dev::ld_rand(a.lidx + v);
}

// Block sum of two int64 per thread (every thread gets both sums).
__device__ __forceinline__ void block_sum2(int64_t& x, int64_t& y, int64_t (*red)[2]) {
    for (int d = 16; d > 0; d >>= 1) {
        x += __shfl_xor_sync(0xffffffffu, x, d);
        y += __shfl_xor_sync(0xffffffffu, y, d);
    }
    if ((threadIdx.x & 31) == 0) {
        red[threadIdx.x >> 5][0] = x;
        red[threadIdx.x >> 5][1] = y;
    }
    __syncthreads();
    x = y = 0;
    for (int w = 0; w < kSampleTile / 32; w++) {
        x += red[w][0];
        y += red[w][1];
    }
}

// All hops' offsets and src in one wait-free pass: a tile's first edge position is the sum of the edge
// counts of the tiles before it, which the hop kernels accumulated per tile (no chained scan, no waiting
// on other blocks); the hop's base is the sum over the earlier hops' tiles.
// 6 blocks/SM minimum (<= 40 registers, 6 slots in flight per thread; its grid is capped at 2 blocks/SM):
// round 1 held it at 64 registers (8 slots: spilled at 40), round 2 measured the smaller footprint faster once
// many lanes' kernels compete for the register files (see MOMENT_SCAN_MINB)
#ifndef MOMENT_COMPACT_MINB
#define MOMENT_COMPACT_MINB 6  // 40 registers (see MOMENT_SCAN_MINB)
#endif
#ifndef MOMENT_COMPACT_UNROLL
#define MOMENT_COMPACT_UNROLL 6  // 8 spills at 40 registers
#endif
__global__ void __launch_bounds__(kSampleTile, MOMENT_COMPACT_MINB) compact_kernel(CompactArgs a) {
    constexpr int kCopyUnroll = MOMENT_COMPACT_UNROLL;  // padded slots per thread in flight (id -> rel / lidx -> src)
    __shared__ int64_t s_red[kSampleTile / 32];
    __shared__ int64_t s_red2[kSampleTile / 32][2];
    __shared__ int32_t s_excl[kSampleTile], s_cnt[kSampleTile];
    const int64_t n_tiles = a.tb[a.H];
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        // hops with an empty frontier have no tile: write their (empty) offsets and E_h here
        int64_t ob = 0;
        for (int h = 0; h < a.H; h++) {
            if (a.counts[h] == 0) {
                a.offsets[ob] = 0;
                a.counts[a.H + 1 + h] = 0;
            }
            ob += a.counts[h] + 1;
        }
    }
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        int h = 0;
        while (tile >= a.tb[h + 1]) h++;
        const int64_t F = a.counts[h];
        const int64_t lt = tile - a.tb[h];
        if (lt * kSampleTile >= F) continue;  // past this hop's frontier (uniform per block)
        int64_t ob = 0;
        for (int q = 0; q < h; q++) ob += a.counts[q] + 1;
        const int64_t idx = lt * kSampleTile + threadIdx.x;
        const int32_t c = idx < F ? a.cnt[h][idx] : 0;
        int64_t before_hop = 0, in_hop = 0;  // edges of the earlier hops' tiles / of this hop's earlier tiles
        for (int64_t j = threadIdx.x; j < tile; j += kSampleTile) {
            const int64_t e = (int64_t)__ldcg(a.tile_edges + j);
            if (j < a.tb[h]) before_hop += e;
            else in_hop += e;
        }
        block_sum2(before_hop, in_hop, s_red2);
        int64_t agg;
        const int64_t excl = dev::block_exclusive_scan<kSampleTile>(c, &agg, s_red);
        const int64_t gpos = before_hop + in_hop + excl;  // global position of this node's first edge
        const int64_t rel = in_hop + excl;
        if (idx < F) {
            a.offsets[ob + idx] = rel;
            if (idx == F - 1) {
                a.offsets[ob + F] = rel + c;
                a.counts[a.H + 1 + h] = rel + c;
            }
        }
        // copy + relabel the tile's edges slot-parallel: the tile's padded rows (nodes x k ints) are read
        // coalesced, slot s belongs to node s / k at rank s % k and is an edge iff its rank < the node's
        // count; kCopyUnroll independent lidx loads in flight per thread
        s_excl[threadIdx.x] = (int32_t)excl;
        s_cnt[threadIdx.x] = c;
        __syncthreads();
        {
            const int k = a.k[h];
            const uint32_t km = a.kmagic[h];
            const int32_t* p = a.pad[h] + lt * kSampleTile * k;
            int32_t* out = a.src + (gpos - excl);  // the tile's first edge
            const int slots = (int)min((int64_t)kSampleTile, F - lt * kSampleTile) * k;
            for (int s0 = threadIdx.x; s0 < slots; s0 += kSampleTile * kCopyUnroll) {
                int32_t id[kCopyUnroll], at[kCopyUnroll];
#pragma unroll
                for (int u = 0; u < kCopyUnroll; u++) {
                    const int sl = s0 + u * kSampleTile;
                    at[u] = -1;
                    if (sl < slots) {
                        const int node = k == 1 ? sl : (int)__umulhi((uint32_t)sl, km);
                        const int r = sl - node * k;
                        if (r < s_cnt[node]) {
                            at[u] = s_excl[node] + r;
                            id[u] = __ldg(p + sl);
                        }
                    }
                }
                if (a.rel) {
                    // first probe (hop h, where most targets are new) for all kCopyUnroll slots in flight
                    const uint2* rel_h = a.rel + h * a.rel_stride;
                    uint2 r[kCopyUnroll];
#pragma unroll
                    for (int u = 0; u < kCopyUnroll; u++)
                        r[u] = at[u] >= 0 ? __ldcg(rel_h + (id[u] >> 5)) : make_uint2(0u, 0u);
                    const int64_t Fh = a.counts[h];
#pragma unroll
                    for (int u = 0; u < kCopyUnroll; u++) {
                        if (at[u] < 0) continue;
                        const uint32_t bit = 1u << (id[u] & 31);
                        id[u] = (r[u].x & bit) ? (int32_t)(Fh + r[u].y + __popc(r[u].x & (bit - 1)))
                                               : rel_position(a, id[u], h - 1);
                    }
                } else if (a.srel) {
                    // two dependent L2 loads per probe (summary-level then entry); 8 slots in flight
                    const uint2* s_h = a.srel + h * a.srel_stride;
                    uint2 m[kCopyUnroll];
#pragma unroll
                    for (int u = 0; u < kCopyUnroll; u++)
                        m[u] = at[u] >= 0 ? __ldcg(s_h + ((uint32_t)id[u] >> 10)) : make_uint2(0u, 0u);
                    uint2 r[kCopyUnroll];
#pragma unroll
                    for (int u = 0; u < kCopyUnroll; u++) {
                        const uint32_t j = ((uint32_t)id[u] >> 5) & 31;
                        r[u] = (at[u] >= 0 && ((m[u].x >> j) & 1u))
                                   ? __ldcg(a.trel[h] + m[u].y + __popc(m[u].x & ((1u << j) - 1u)))
                                   : make_uint2(0u, 0u);
                    }
                    const int64_t Fh = a.counts[h];
#pragma unroll
                    for (int u = 0; u < kCopyUnroll; u++) {
                        if (at[u] < 0) continue;
                        const uint32_t bit = 1u << (id[u] & 31);
                        id[u] = (r[u].x & bit) ? (int32_t)(Fh + r[u].y + __popc(r[u].x & (bit - 1)))
                                               : rel_position(a, id[u], h - 1);
                    }
                } else {
#pragma unroll
                    for (int u = 0; u < kCopyUnroll; u++) id[u] = at[u] >= 0 ? dev::ld_rand(a.lidx + id[u]) : 0;
                }
#pragma unroll
                for (int u = 0; u < kCopyUnroll; u++)
                    if (at[u] >= 0) out[at[u]] = id[u];
            }
        }
        __syncthreads();  // s_red / s_red2 / s_excl / s_cnt are reused by the next tile
    }
    // moment_step_host with mapped host counts: the last block to finish stores the call's 2H + 1 counts into
    // host memory (every block's writes are visible to it: fence, then the done-counter ticket)
    if (a.call && a.call[2]) {
        __shared__ bool s_last;
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            s_last = atomicAdd(a.done, 1u) == gridDim.x - 1;
        }
        __syncthreads();
        if (s_last && threadIdx.x < 2 * a.H + 1) {
            __threadfence();
            reinterpret_cast<volatile int64_t*>(a.call[2])[threadIdx.x] = *reinterpret_cast<volatile int64_t*>(a.counts + threadIdx.x);
        }
    }
    if (!a.visited) return;  // cleared by a memset after the kernel instead (MOMENT_VISITED_MEMSET)
    const int64_t FH = a.counts[a.H];
    for (int64_t i = (int64_t)blockIdx.x * kSampleTile + threadIdx.x; i < FH; i += (int64_t)gridDim.x * kSampleTile)
        a.visited[a.nodes[i] >> 5] = 0u;
}

__global__ void init_kernel(const uint64_t* call, int64_t n_seeds, int64_t n_vertices, int64_t* nodes, int32_t* lidx,
                            uint32_t* visited, int64_t* counts, uint32_t* error_flag, int check, uint64_t* tile_status,
                            int64_t n_tile_status, uint32_t* tickets, int n_tickets, uint64_t* ebase, int n_ebase) {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (int64_t)gridDim.x * blockDim.x;
    const int64_t* seeds = reinterpret_cast<const int64_t*>(call[1]);
    for (int64_t i = tid; i < n_tile_status; i += nth) tile_status[i] = 0;
    for (int64_t i = tid; i < n_tickets; i += nth) tickets[i] = 0;
    for (int64_t i = tid; i < n_ebase; i += nth) ebase[i] = 0;
    for (int64_t i = tid; i < n_seeds; i += nth) {
        const int64_t v = seeds[i];
        if (v < 0 || v >= n_vertices) {  // never write out of range, checked or not
            atomicOr(error_flag, 1u);
            nodes[i] = 0;
            continue;
        }
        nodes[i] = v;
        lidx[v] = (int32_t)i;
        const uint32_t bit = 1u << (v & 31);
        const uint32_t old = atomicOr(visited + (v >> 5), bit);
        if (check && (old & bit)) atomicOr(error_flag, 2u);
    }
    if (tid == 0) counts[0] = n_seeds;
}

template <int G, int Q>
void launch_sample_hop_q(const HopArgs& a, int64_t max_F, cudaStream_t stream) {
    const int64_t groups = (max_F + Q - 1) / Q;
    const int64_t blocks = std::max<int64_t>(1, (groups * G + 255) / 256);
    hop_sample_kernel<G, Q><<<(int)std::min<int64_t>(blocks, (int64_t)device_sms() * a.grid_per_sm), 256, 0, stream>>>(a);
}

// Small frontiers keep one node per group (latency: every node in flight at once); large frontiers batch
// `big_q` nodes per group (throughput: that many chains in flight per thread, 1/big_q of the warps).
template <int G>
void launch_sample_hop(const HopArgs& a, int64_t max_F, int big_q, cudaStream_t stream) {
    if (max_F < 65536 || big_q <= 1) launch_sample_hop_q<G, 1>(a, max_F, stream);
    else if (big_q <= 2) launch_sample_hop_q<G, 2>(a, max_F, stream);
    else if (big_q <= 4) launch_sample_hop_q<G, 4>(a, max_F, stream);
    else launch_sample_hop_q<G, 8>(a, max_F, stream);
}

template <int Q, bool kInit = false>
void launch_sample_warp_q(const HopArgs& a, int64_t max_F, cudaStream_t stream, const InitArgs& in = InitArgs{}) {
    const int64_t per_warp = (int64_t)(32 / a.k) * Q;
    const int64_t warps = (max_F + per_warp - 1) / per_warp;
    const int64_t blocks = std::max<int64_t>(1, (warps + 7) / 8);
    hop_sample_warp_kernel<Q, kInit>
        <<<(int)std::min<int64_t>(blocks, (int64_t)device_sms() * a.grid_per_sm), 256, 0, stream>>>(a, in);
}

#ifndef MOMENT_HOP_BIG_F
// frontier bound from which a lane group takes big_q nodes per step: C2's and C3's hops 1 and 2 (bounds 16 k and
// 180 k); round 2: lowered from 65536 (hop 2 only), C2 step 24.65 -> 23.95 us, C3 89.0 -> 86.9 us at 16 lanes
#define MOMENT_HOP_BIG_F 8192
#endif
void launch_sample_warp(const HopArgs& a, int64_t max_F, int big_q, cudaStream_t stream) {
    if (max_F < MOMENT_HOP_BIG_F || big_q <= 1) launch_sample_warp_q<1>(a, max_F, stream);
    else if (big_q <= 2) launch_sample_warp_q<2>(a, max_F, stream);
    else launch_sample_warp_q<4>(a, max_F, stream);
}

}  // namespace

// Same shared-memory carveout for every kernel of the library (see configure_gather_kernels).
moment_status configure_sample_kernels(int carveout) {
    if (carveout < 0) return MOMENT_OK;
    const void* fns[] = {(const void*)init_kernel, (const void*)bitscan_kernel<false>, (const void*)bitscan_kernel<true>,
                         (const void*)bitscan_sparse_kernel<256>,
                         (const void*)bitscan_sparse_kernel<512>, (const void*)bitscan_sparse_kernel<1024>,
                         (const void*)compact_kernel,
                         (const void*)hop_sample_kernel<4, 1>, (const void*)hop_sample_kernel<8, 1>,
                         (const void*)hop_sample_kernel<16, 1>, (const void*)hop_sample_kernel<32, 1>,
                         (const void*)hop_sample_kernel<4, 2>, (const void*)hop_sample_kernel<8, 2>,
                         (const void*)hop_sample_kernel<16, 2>, (const void*)hop_sample_kernel<32, 2>,
                         (const void*)hop_sample_kernel<4, 4>, (const void*)hop_sample_kernel<8, 4>,
                         (const void*)hop_sample_kernel<16, 4>, (const void*)hop_sample_kernel<32, 4>,
                         (const void*)hop_sample_kernel<4, 8>, (const void*)hop_sample_kernel<8, 8>,
                         (const void*)hop_sample_kernel<16, 8>, (const void*)hop_sample_kernel<32, 8>,
                         (const void*)hop_sample_warp_kernel<1, false>, (const void*)hop_sample_warp_kernel<2, false>,
                         (const void*)hop_sample_warp_kernel<4, false>, (const void*)hop_sample_warp_kernel<1, true>};
    for (const void* f : fns)
        MOMENT_TRY(cuda_check(cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, carveout),
                              "carveout attribute"));
    return MOMENT_OK;
}

// Validates the call on the host; enqueues nothing on error. The seeds pointer and rng_seed are read by
// the kernels from the device call block `call` ([0] rng_seed, [1] seeds), written beforehand by the
// caller (ctx.cu) so that a captured graph of these launches serves every batch.
moment_status check_sample(const moment_ctx_s* ctx, const moment_csr* csr, const int64_t* seeds, int64_t n_seeds,
                           const moment_sample_params* p, const moment_sample_out* out) {
    if (!csr || !p || !out || (!seeds && n_seeds > 0)) return fail(MOMENT_EINVAL, "moment_sample: null argument");
    if (csr->n_vertices != ctx->n_vertices || !csr->indptr || !csr->indices)
        return fail(MOMENT_EINVAL, "moment_sample: csr has %lld vertices, ctx was created for %lld",
                    (long long)csr->n_vertices, (long long)ctx->n_vertices);
    // n_edges picks the launch variant (the bitscan's neighbour prefetch) and must describe `indices`;
    // indptr[n] == n_edges is the caller's contract (checking it would need a device read)
    if (csr->n_edges < 0 || csr->n_edges >= (int64_t(1) << 40))
        return fail(MOMENT_EINVAL, "moment_sample: n_edges %lld out of range", (long long)csr->n_edges);
    const int H = p->n_hops;
    if (H < 0 || H > ctx->max_hops || H > kMaxHops)
        return fail(MOMENT_EINVAL, "moment_sample: n_hops %d > max_hops %d", H, ctx->max_hops);
    if (n_seeds < 0 || n_seeds > ctx->max_seeds)
        return fail(MOMENT_EINVAL, "moment_sample: n_seeds %lld > max_seeds %lld", (long long)n_seeds, (long long)ctx->max_seeds);
    if (H > 0 && !p->fanout) return fail(MOMENT_EINVAL, "moment_sample: fanout is null");
    for (int h = 0; h < H; h++)
        if (p->fanout[h] < 1 || p->fanout[h] > ctx->max_fanout[h] || p->fanout[h] > kMaxFanout)
            return fail(MOMENT_EINVAL, "moment_sample: fanout[%d] = %d outside [1, %d]", h, p->fanout[h],
                        std::min(ctx->max_fanout[h], kMaxFanout));
    int64_t need_nodes, need_offsets, need_edges;
    MOMENT_TRY(moment_sample_bounds(n_seeds, p->fanout, H, ctx->n_vertices, &need_nodes, &need_offsets, &need_edges));
    if (!out->nodes || !out->counts || (H > 0 && (!out->offsets || !out->src)))
        return fail(MOMENT_EINVAL, "moment_sample: null output buffer");
    if (out->cap_nodes < need_nodes || out->cap_offsets < need_offsets || out->cap_edges < need_edges)
        return fail(MOMENT_EOVERFLOW, "moment_sample: output capacity too small: need nodes %lld offsets %lld edges %lld",
                    (long long)need_nodes, (long long)need_offsets, (long long)need_edges);
    return cuda_pending("moment_sample: pending CUDA error");
}

// Enqueues the 2H + 2 kernels of one sample call (arguments already validated by check_sample).
moment_status launch_sample(moment_ctx_s* ctx, const moment_csr* csr, const uint64_t* call, int64_t n_seeds,
                            const moment_sample_params* p, const moment_sample_out* out, cudaStream_t stream,
                            cudaEvent_t after_hops) {
    const int H = p->n_hops;
    const int check = (p->flags & MOMENT_SAMPLE_CHECK) ? 1 : 0;
    const int replace = (p->flags & MOMENT_SAMPLE_REPLACE) ? 1 : 0;
    // the first hop initialises the call itself when it runs the warp-segmented sampler (one launch fewer)
    const bool init_in_hop0 = H > 0 && ctx->hop_warp_segmented && p->fanout[0] <= 32 && ctx->init_in_hop0;
    const InitArgs init{n_seeds, ctx->n_vertices, out->nodes, out->counts, ctx->lidx, ctx->visited, ctx->error_flag,
                        check, ctx->tile_status, ctx->n_tile_status, ctx->tickets, 1 + std::max(1, ctx->max_hops),
                        ctx->ebase, std::max(1, ctx->max_hops)};
    if (!init_in_hop0) {
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((n_seeds + 255) / 256, device_sms() * 4));
        init_kernel<<<grid, 256, 0, stream>>>(call, n_seeds, ctx->n_vertices, out->nodes, ctx->lidx, ctx->visited,
                                              out->counts, ctx->error_flag, check, ctx->tile_status, ctx->n_tile_status,
                                              ctx->tickets, 1 + std::max(1, ctx->max_hops), ctx->ebase,
                                              std::max(1, ctx->max_hops));
    }
    // per-call bounds on |F_h| for launch sizing, padded-buffer carving and compaction tile numbering (the
    // true sizes live in counts); hop h's tile sums are tile_edges[tb[h] .. tb[h + 1])
    CompactArgs ca{};
    {
        int64_t Fb = n_seeds;
        ca.tb[0] = 0;
        for (int h = 0; h < H; h++) {
            ca.tb[h + 1] = ca.tb[h] + (Fb + kSampleTile - 1) / kSampleTile;
            Fb = std::min(Fb + Fb * (int64_t)p->fanout[h], ctx->n_vertices);
        }
    }
    int64_t F_bound = n_seeds, pad_off = 0, cnt_off = 0;
    const int64_t n_scan_tiles = (ctx->n_words + kScanTileWords - 1) / kScanTileWords;
    for (int h = 0; h < H; h++) {
        const int k = p->fanout[h];
        HopArgs a{csr->indptr, csr->indices, out->nodes, out->counts, ctx->pad + pad_off, ctx->cnt + cnt_off,
                  ctx->newbits, ctx->sparse_scan ? ctx->summary : nullptr, call, h, k, replace,
                  ctx->hop_grid_per_sm, ctx->tile_edges + ca.tb[h], h + 1 < H ? (ctx->hop_prefetch > 0 ? ctx->hop_prefetch : (ctx->hop_prefetch < 0 && !ctx->sparse_scan)) : 0};
        const int q = ctx->hop_nodes_per_group;
        if (h == 0 && init_in_hop0) launch_sample_warp_q<1, true>(a, F_bound, stream, init);
        else if (ctx->hop_warp_segmented && k <= 32) launch_sample_warp(a, F_bound, q, stream);
        else if (k <= 4) launch_sample_hop<4>(a, F_bound, q, stream);
        else if (k <= 8) launch_sample_hop<8>(a, F_bound, q, stream);
        else if (k <= 16) launch_sample_hop<16>(a, F_bound, q, stream);
        else launch_sample_hop<32>(a, F_bound, q, stream);
        const int64_t n_zero = h + 1 < H ? ca.tb[h + 2] - ca.tb[h + 1] : 0;  // the next hop's tile sums
        uint2* rel = (ctx->rel && !ctx->sparse_scan) ? ctx->rel + (int64_t)h * ctx->rel_stride : nullptr;
        uint2* srel = ctx->srel ? ctx->srel + (int64_t)h * ctx->srel_stride : nullptr;
        uint2* trel = ctx->srel ? ctx->trel + ctx->trel_off[h] : nullptr;
        ScanArgs s{out->nodes, out->counts, ctx->lidx, ctx->newbits, ctx->visited, ctx->summary,
                   ctx->tile_status + ctx->bitscan_tiles_off[h], ctx->tickets + 1 + h, ctx->n_words, h,
                   ctx->tile_edges + ca.tb[h + 1], n_zero, rel, srel, trel, csr->indptr, csr->indices,
                   !ctx->sparse_scan && h + 1 < H &&
                       (ctx->scan_prefetch > 0 || (ctx->scan_prefetch < 0 && csr->n_edges <= kScanPrefetchMaxEdges))};
        if (srel) ca.trel[h] = trel;
        if (ctx->sparse_scan) {  // one summary word (32 newbits words) per thread
            const int nt = ctx->sparse_threads;
            const int64_t tiles = (ctx->n_words + 32 * nt - 1) / (32 * nt);
            const int grid = (int)std::min<int64_t>(tiles, device_sms() * (1024 / nt) * 2);
            if (nt == 1024) bitscan_sparse_kernel<1024><<<grid, 1024, 0, stream>>>(s);
            else if (nt == 512) bitscan_sparse_kernel<512><<<grid, 512, 0, stream>>>(s);
            else bitscan_sparse_kernel<256><<<grid, 256, 0, stream>>>(s);
        } else {
            const int nb = (int)std::min<int64_t>(n_scan_tiles, device_sms() * 4);
            if (s.prefetch_idx) bitscan_kernel<true><<<nb, kBitscanThreads, 0, stream>>>(s);
            else bitscan_kernel<false><<<nb, kBitscanThreads, 0, stream>>>(s);
        }
        ca.k[h] = k;
        ca.kmagic[h] = k == 1 ? 0u : (uint32_t)(((uint64_t(1) << 32) + (uint64_t)k - 1) / (uint64_t)k);
        ca.pad[h] = ctx->pad + pad_off;
        ca.cnt[h] = ctx->cnt + cnt_off;
        pad_off += F_bound * k;
        cnt_off += F_bound;
        F_bound = std::min(F_bound + F_bound * (int64_t)k, ctx->n_vertices);
    }
    if (after_hops) MOMENT_TRY(cuda_check(cudaEventRecord(after_hops, stream), "moment_sample: fork event"));
    ca.offsets = out->offsets;
    ca.src = out->src;
    ca.counts = out->counts;
    ca.nodes = out->nodes;
    ca.lidx = ctx->lidx;
    ca.visited = ctx->visited_memset ? nullptr : ctx->visited;
    ca.rel = ctx->sparse_scan ? nullptr : ctx->rel;
    ca.rel_stride = ctx->rel_stride;
    ca.srel = ctx->srel;
    ca.srel_stride = ctx->srel_stride;
    ca.tile_edges = ctx->tile_edges;
    ca.H = H;
    ca.call = call;
    ca.done = ctx->tickets;  // tickets[0]: compaction blocks done (zeroed by the call's init)
    const int grid = (int)std::max<int64_t>(
        1, std::min<int64_t>(std::max(ca.tb[H], (F_bound + 1023) / 1024), (int64_t)device_sms() * ctx->compact_grid_per_sm));
    compact_kernel<<<grid, kSampleTile, 0, stream>>>(ca);
    if (ctx->visited_memset)
        MOMENT_TRY(cuda_check(cudaMemsetAsync(ctx->visited, 0, (size_t)ctx->n_words * sizeof(uint32_t), stream),
                              "moment_sample: visited reset"));
    return cuda_check(cudaGetLastError(), "moment_sample: launch");
}

}  // namespace moment

extern "C" moment_status moment_sample_bounds(int64_t n_seeds, const int32_t* fanout, int32_t n_hops, int64_t n_vertices,
                                              int64_t* max_nodes, int64_t* max_offsets, int64_t* max_edges) {
    if (n_seeds < 0 || n_hops < 0 || n_vertices <= 0 || (n_hops > 0 && !fanout))
        return moment::fail(MOMENT_EINVAL, "moment_sample_bounds: bad argument");
    int64_t F = std::min(n_seeds, n_vertices), E = 0, O = 0;
    for (int h = 0; h < n_hops; h++) {
        if (fanout[h] < 1) return moment::fail(MOMENT_EINVAL, "moment_sample_bounds: fanout[%d] = %d", h, fanout[h]);
        O += F + 1;
        E += F * (int64_t)fanout[h];
        F = std::min(F + F * (int64_t)fanout[h], n_vertices);
    }
    if (max_nodes) *max_nodes = std::max<int64_t>(F, n_seeds);
    if (max_offsets) *max_offsets = O;
    if (max_edges) *max_edges = E;
    return MOMENT_OK;
}
