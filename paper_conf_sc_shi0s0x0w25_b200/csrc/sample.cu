// sample.cu — H1-H3: multi-hop neighbour sampling with dedup/relabel on sm_100a (R3-R6).
//
// Per hop h the path is three kernels, none of which needs the host to know |F_h| or E_h (every size is
// read from device memory, so the whole sample call is CUDA-graph capturable):
//   sample_hop  : tile of 256 frontier nodes -> degrees -> block scan + decoupled look-back = edge offsets;
//                 then one G-lane group per node draws its Floyd / with-replacement positions from
//                 Philox, writes the neighbour ids and marks them in the `newbits` bitmap.
//   bitscan     : F_{h+1} = F_h ++ (newbits & ~visited) in ascending id order: a chained scan of bitmap
//                 popcounts (2048 words per tile) gives each new id its position; lidx[id] = position.
//   relabel     : src[e] = lidx[src[e]] (global id -> index in F_{h+1}).
#include <cooperative_groups.h>

#include <algorithm>

#include "ctx.h"
#include "device_util.cuh"

namespace cg = cooperative_groups;

namespace moment {
namespace {

struct HopArgs {
    const int64_t* indptr;
    const int32_t* indices;
    int64_t* nodes;
    int64_t* offsets;
    int32_t* src;
    int64_t* counts;
    uint32_t* newbits;
    uint64_t* tile_status;
    uint32_t* ticket;
    uint64_t seed;
    int32_t h, H, k;
    int32_t replace;
};

// Sizes of earlier hops live in counts: offsets block h starts at sum_{h'<h} (|F_h'| + 1) and the
// edges of hop h at sum_{h'<h} E_h'.
__device__ __forceinline__ void hop_bases(const int64_t* counts, int h, int H, int64_t* off_base, int64_t* edge_base) {
    int64_t ob = 0, eb = 0;
    for (int q = 0; q < h; q++) {
        ob += counts[q] + 1;
        eb += counts[H + 1 + q];
    }
    *off_base = ob;
    *edge_base = eb;
}

__device__ __forceinline__ void mark_new(uint32_t* newbits, int32_t u) {
    const uint32_t bit = 1u << (u & 31);
    uint32_t* w = newbits + (u >> 5);
    if ((__ldcg(w) & bit) == 0) atomicOr(w, bit);
}

// One node, one group of G lanes. Positions are distinct CSR offsets in [0, d).
template <int G>
__device__ __forceinline__ void sample_node(const cg::thread_block_tile<G>& grp, const HopArgs& a, int64_t v,
                                            int64_t lo, int32_t d, int32_t* out) {
    const int lane = grp.thread_rank();
    const int k = a.k;
    if (d <= 0) return;
    if (a.replace) {
        // with replacement: k draws in draw order
        for (int i = lane; i < k; i += G) {
            const uint32_t p = dev::uniform(dev::draw(a.seed, v, a.h, i), (uint32_t)d);
            const int32_t u = __ldg(a.indices + lo + p);
            out[i] = u;
            mark_new(a.newbits, u);
        }
        return;
    }
    if (d <= k) {
        // take all neighbours, CSR order, no draws
        for (int p = lane; p < d; p += G) {
            const int32_t u = __ldg(a.indices + lo + p);
            out[p] = u;
            mark_new(a.newbits, u);
        }
        return;
    }
    if (k <= G) {
        // Floyd F2 with the k choices resolved in draw order by group ballots; lane i owns choice i.
        int32_t j = 0, t = 0, c = -1;
        if (lane < k) {
            j = d - k + lane;
            t = (int32_t)dev::uniform(dev::draw(a.seed, v, a.h, lane), (uint32_t)(j + 1));
        }
        for (int m = 0; m < k; m++) {
            const int32_t tm = grp.shfl(t, m);
            const bool hit = lane < m && c == tm;
            const unsigned any = grp.ballot(hit);
            if (lane == m) c = any ? j : t;
        }
        // rank of c among the k distinct choices = its position in sorted order
        int r = 0;
        for (int l = 0; l < k; l++) r += grp.shfl(c, l) < c;
        if (lane < k) {
            const int32_t u = __ldg(a.indices + lo + c);
            out[r] = u;
            mark_new(a.newbits, u);
        }
        return;
    }
    // k > G (only G == 32 reaches here): chunks of 32 choices; earlier chunks are final and kept in
    // `out` as positions, then replaced by ids after the sort.
    for (int c0 = 0; c0 < k; c0 += G) {
        const int i = c0 + lane;
        int32_t j = 0, t = 0, c = -1;
        bool prev_hit = false;
        if (i < k) {
            j = d - k + i;
            t = (int32_t)dev::uniform(dev::draw(a.seed, v, a.h, i), (uint32_t)(j + 1));
            for (int q = 0; q < c0; q++) prev_hit |= out[q] == t;
        }
        const int nm = min(G, k - c0);
        for (int m = 0; m < nm; m++) {
            const int32_t tm = grp.shfl(t, m);
            const bool hit = lane < m && c == tm;
            const unsigned any = grp.ballot(hit);
            if (lane == m) c = (any || prev_hit) ? j : t;
        }
        grp.sync();
        if (i < k) out[i] = c;
        grp.sync();
    }
    // sort positions: rank by counting (distinct), then write ids
    int32_t mine[kMaxFanout / 32];
    int rk[kMaxFanout / 32];
    const int per = (k + G - 1) / G;
    for (int q = 0; q < per; q++) {
        const int i = q * G + lane;
        mine[q] = i < k ? out[i] : 0;
        int r = 0;
        if (i < k)
            for (int l = 0; l < k; l++) r += out[l] < mine[q];
        rk[q] = r;
    }
    grp.sync();
    for (int q = 0; q < per; q++) {
        const int i = q * G + lane;
        if (i < k) {
            const int32_t u = __ldg(a.indices + lo + mine[q]);
            out[rk[q]] = u;
            mark_new(a.newbits, u);
        }
    }
}

template <int G>
__global__ void __launch_bounds__(kSampleTile) sample_hop_kernel(HopArgs a) {
    __shared__ int64_t s_v[kSampleTile], s_lo[kSampleTile], s_off[kSampleTile];
    __shared__ int32_t s_deg[kSampleTile];
    __shared__ int64_t s_warp[kSampleTile / 32];
    __shared__ int64_t s_prefix;
    __shared__ uint32_t s_tile;
    const int64_t F = a.counts[a.h];
    int64_t off_base, edge_base;
    hop_bases(a.counts, a.h, a.H, &off_base, &edge_base);
    int64_t* offsets = a.offsets + off_base;
    int32_t* src = a.src + edge_base;
    const int64_t n_tiles = (F + kSampleTile - 1) / kSampleTile;
    if (F == 0) {
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            offsets[0] = 0;
            a.counts[a.H + 1 + a.h] = 0;
        }
        return;
    }
    auto grp = cg::tiled_partition<G>(cg::this_thread_block());
    const int group = threadIdx.x / G, n_groups = kSampleTile / G;
    for (;;) {
        if (threadIdx.x == 0) s_tile = atomicAdd(a.ticket, 1u);
        __syncthreads();
        const int64_t tile = s_tile;
        if (tile >= n_tiles) break;
        const int64_t idx = tile * kSampleTile + threadIdx.x;
        int64_t v = 0, lo = 0;
        int32_t d = 0, c = 0;
        if (idx < F) {
            v = a.nodes[idx];
            lo = __ldg(a.indptr + v);
            d = (int32_t)(__ldg(a.indptr + v + 1) - lo);
            c = a.replace ? (d > 0 ? a.k : 0) : min(d, a.k);
        }
        int64_t agg;
        const int64_t excl = dev::block_exclusive_scan<kSampleTile>(c, &agg, s_warp);
        if (threadIdx.x == 0) s_prefix = dev::lookback(a.tile_status, tile, agg);
        __syncthreads();
        const int64_t off = s_prefix + excl;
        if (idx < F) {
            offsets[idx] = off;
            if (idx == F - 1) {
                offsets[F] = off + c;
                a.counts[a.H + 1 + a.h] = off + c;
            }
        }
        s_v[threadIdx.x] = v;
        s_lo[threadIdx.x] = lo;
        s_deg[threadIdx.x] = d;
        s_off[threadIdx.x] = off;
        __syncthreads();
        const int live = (int)min((int64_t)kSampleTile, F - tile * kSampleTile);
        for (int j = group; j < live; j += n_groups) sample_node<G>(grp, a, s_v[j], s_lo[j], s_deg[j], src + s_off[j]);
        __syncthreads();
    }
}

struct ScanArgs {
    int64_t* nodes;
    int64_t* counts;
    int32_t* lidx;
    uint32_t* newbits;
    uint32_t* visited;
    uint64_t* tile_status;
    uint32_t* ticket;
    int64_t n_words;
    int32_t h;
};

// F_{h+1} = F_h ++ ascending ids set in (newbits & ~visited).
__global__ void __launch_bounds__(kBitscanThreads) bitscan_kernel(ScanArgs a) {
    __shared__ int64_t s_warp[kBitscanThreads / 32];
    __shared__ int64_t s_prefix;
    __shared__ uint32_t s_tile;
    const int64_t F = a.counts[a.h];
    const int64_t n_tiles = (a.n_words + kBitscanTileWords - 1) / kBitscanTileWords;
    for (;;) {
        if (threadIdx.x == 0) s_tile = atomicAdd(a.ticket, 1u);
        __syncthreads();
        const int64_t tile = s_tile;
        if (tile >= n_tiles) break;
        const int64_t w0 = tile * kBitscanTileWords + (int64_t)threadIdx.x * kBitscanWordsPerThread;
        uint32_t nb[kBitscanWordsPerThread], nw[kBitscanWordsPerThread];
        int cnt = 0;
        if (w0 + kBitscanWordsPerThread <= a.n_words) {
            const uint4* pn = reinterpret_cast<const uint4*>(a.newbits + w0);
            const uint4* pv = reinterpret_cast<const uint4*>(a.visited + w0);
            uint4 n0 = __ldcg(pn), n1 = __ldcg(pn + 1), v0 = __ldcg(pv), v1 = __ldcg(pv + 1);
            nb[0] = n0.x; nb[1] = n0.y; nb[2] = n0.z; nb[3] = n0.w; nb[4] = n1.x; nb[5] = n1.y; nb[6] = n1.z; nb[7] = n1.w;
            uint32_t vv[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
#pragma unroll
            for (int q = 0; q < 8; q++) {
                nw[q] = nb[q] & ~vv[q];
                cnt += __popc(nw[q]);
            }
        } else {
#pragma unroll
            for (int q = 0; q < 8; q++) {
                const int64_t w = w0 + q;
                nb[q] = w < a.n_words ? __ldcg(a.newbits + w) : 0u;
                nw[q] = w < a.n_words ? nb[q] & ~__ldcg(a.visited + w) : 0u;
                cnt += __popc(nw[q]);
            }
        }
        int64_t agg;
        const int64_t excl = dev::block_exclusive_scan<kBitscanThreads>(cnt, &agg, s_warp);
        if (threadIdx.x == 0) s_prefix = dev::lookback(a.tile_status, tile, agg);
        __syncthreads();
        int64_t pos = F + s_prefix + excl;
        if (tile == n_tiles - 1 && threadIdx.x == 0) a.counts[a.h + 1] = F + s_prefix + agg;
#pragma unroll
        for (int q = 0; q < 8; q++) {
            const int64_t w = w0 + q;
            uint32_t bits = nw[q];
            while (bits) {
                const int b = __ffs(bits) - 1;
                bits &= bits - 1;
                const int64_t id = w * 32 + b;
                a.nodes[pos] = id;
                a.lidx[id] = (int32_t)pos;
                pos++;
            }
            if (nb[q]) {
                a.newbits[w] = 0u;
                a.visited[w] |= nw[q];
            }
        }
        __syncthreads();
    }
}

__global__ void relabel_kernel(int32_t* src_all, const int64_t* counts, const int32_t* lidx, int h, int H) {
    int64_t off_base, edge_base;
    hop_bases(counts, h, H, &off_base, &edge_base);
    const int64_t E = counts[H + 1 + h];
    int32_t* src = src_all + edge_base;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x)
        src[e] = __ldg(lidx + src[e]);
}

__global__ void init_seeds_kernel(const int64_t* seeds, int64_t n_seeds, int64_t n_vertices, int64_t* nodes,
                                  int32_t* lidx, uint32_t* visited, int64_t* counts, uint32_t* error_flag,
                                  int check) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n_seeds; i += (int64_t)gridDim.x * blockDim.x) {
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
    if (blockIdx.x == 0 && threadIdx.x == 0) counts[0] = n_seeds;
}

template <int G>
void launch_hop(const HopArgs& a, int64_t max_F, cudaStream_t stream) {
    const int64_t tiles = std::max<int64_t>(1, (max_F + kSampleTile - 1) / kSampleTile);
    const int grid = (int)std::min<int64_t>(tiles, 148 * 8);
    sample_hop_kernel<G><<<grid, kSampleTile, 0, stream>>>(a);
}

}  // namespace

moment_status launch_sample(moment_ctx_s* ctx, const moment_csr* csr, const int64_t* seeds, int64_t n_seeds,
                            const moment_sample_params* p, const moment_sample_out* out, cudaStream_t stream) {
    if (!csr || !p || !out || (!seeds && n_seeds > 0)) return fail(MOMENT_EINVAL, "moment_sample: null argument");
    if (csr->n_vertices != ctx->n_vertices || !csr->indptr || !csr->indices)
        return fail(MOMENT_EINVAL, "moment_sample: csr has %lld vertices, ctx was created for %lld",
                    (long long)csr->n_vertices, (long long)ctx->n_vertices);
    const int H = p->n_hops;
    if (H < 0 || H > ctx->max_hops) return fail(MOMENT_EINVAL, "moment_sample: n_hops %d > max_hops %d", H, ctx->max_hops);
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
    MOMENT_TRY(cuda_pending("moment_sample: pending CUDA error"));
    const int check = (p->flags & MOMENT_SAMPLE_CHECK) ? 1 : 0;
    const int replace = (p->flags & MOMENT_SAMPLE_REPLACE) ? 1 : 0;
    MOMENT_TRY(cuda_check(cudaMemsetAsync(ctx->visited, 0, ctx->n_words * sizeof(uint32_t), stream), "memset visited"));
    MOMENT_TRY(cuda_check(cudaMemsetAsync(ctx->tile_status, 0, ctx->n_tile_status * sizeof(uint64_t), stream), "memset tiles"));
    MOMENT_TRY(cuda_check(cudaMemsetAsync(ctx->tickets, 0, 2 * std::max(1, ctx->max_hops) * sizeof(uint32_t), stream), "memset tickets"));
    {
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((n_seeds + 255) / 256, 148 * 4));
        init_seeds_kernel<<<grid, 256, 0, stream>>>(seeds, n_seeds, ctx->n_vertices, out->nodes, ctx->lidx, ctx->visited,
                                                    out->counts, ctx->error_flag, check);
    }
    // per-call bounds on |F_h| for launch sizing (the kernels read the true sizes from counts)
    int64_t F_bound = n_seeds;
    for (int h = 0; h < H; h++) {
        HopArgs a{csr->indptr, csr->indices, out->nodes, out->offsets, out->src, out->counts, ctx->newbits,
                  ctx->tile_status + ctx->sample_tiles_off[h], ctx->tickets + 2 * h, p->rng_seed, h, H, p->fanout[h], replace};
        const int k = p->fanout[h];
        if (k <= 4) launch_hop<4>(a, F_bound, stream);
        else if (k <= 8) launch_hop<8>(a, F_bound, stream);
        else if (k <= 16) launch_hop<16>(a, F_bound, stream);
        else launch_hop<32>(a, F_bound, stream);
        ScanArgs s{out->nodes, out->counts, ctx->lidx, ctx->newbits, ctx->visited,
                   ctx->tile_status + ctx->bitscan_tiles_off[h], ctx->tickets + 2 * h + 1, ctx->n_words, h};
        const int64_t tiles = (ctx->n_words + kBitscanTileWords - 1) / kBitscanTileWords;
        bitscan_kernel<<<(int)std::min<int64_t>(tiles, 148 * 4), kBitscanThreads, 0, stream>>>(s);
        const int64_t E_bound = F_bound * (int64_t)k;
        const int rgrid = (int)std::max<int64_t>(1, std::min<int64_t>((E_bound + 255) / 256, 148 * 8));
        relabel_kernel<<<rgrid, 256, 0, stream>>>(out->src, out->counts, ctx->lidx, h, H);
        F_bound = std::min(F_bound + F_bound * (int64_t)k, ctx->n_vertices);
    }
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
