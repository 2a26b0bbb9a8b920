// gather.cu — H4-H7 and P2 on sm_100a: placement lookup + bucketing, the 128-bit tiered row gather
// (local HBM / NVLink peer HBM / zero-copy pinned host), the relay of host rows for another rank, and
// the hotness histogram of pre-sampling.
#include <algorithm>

#include "ctx.h"
#include "device_util.cuh"

namespace moment {
namespace {

constexpr int kGatherThreads = 256;
constexpr int kGatherUnroll = 8;  // 16-byte loads in flight per thread
constexpr uint64_t kSlotMask = (1ull << 40) - 1;
constexpr int kMaxQueues = 128;  // n_bins * world

struct BinTable {
    const int4* base[MOMENT_MAX_BINS];  // bin base as addressable from the launching device
    int8_t owner[MOMENT_MAX_BINS];      // owning rank of an HBM bin, -1 for a host-DRAM bin
};

// Row vectors: no L1 allocation, 64-byte L2 fetch size (a row fetches its 64-byte chunks, not whole 128-byte
// lines: profiles/r01_dram_granularity.txt).
__device__ __forceinline__ int4 ld_stream(const int4* p) {
    int4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::64B.v4.s32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
    return r;
}

// Division of a 32-bit index by the runtime row width: q = umulhi64(e, ceil(2^64 / d)) is exact for
// e < 2^32 (Lemire et al., "Faster remainder by direct computation").
struct FastDiv {
    uint64_t m;
    uint32_t d;
};
__device__ __forceinline__ uint32_t fdiv(uint32_t e, const FastDiv& f) {
    return f.d == 1 ? e : (uint32_t)__umul64hi((uint64_t)e, f.m);
}

FastDiv make_fastdiv(uint32_t d) { return FastDiv{d == 1 ? 0ull : (~0ull / d + 1), d}; }

// out[i] = row(ids[i]) for i < n, one 16-byte vector per thread step, kGatherUnroll loads in flight.
// placement == nullptr: replicated table in bin 0 at slot = id. route != nullptr: requests whose route
// says "relay through rank != self" are skipped (the relay rank writes them).
__global__ void __launch_bounds__(kGatherThreads) gather_kernel(BinTable bins, const uint64_t* __restrict__ placement,
                                                                const int64_t* __restrict__ ids, const int64_t* n_dev,
                                                                int64_t max_n, FastDiv rv, int64_t stride_vec,
                                                                const int32_t* __restrict__ route, int32_t world,
                                                                int32_t self, int4* __restrict__ out) {
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    const uint32_t total = (uint32_t)(n * rv.d);
    const uint32_t step = gridDim.x * kGatherThreads * kGatherUnroll;
    for (uint32_t base = blockIdx.x * kGatherThreads * kGatherUnroll + threadIdx.x; base < total; base += step) {
        int4 val[kGatherUnroll];
        bool live[kGatherUnroll];
#pragma unroll
        for (int u = 0; u < kGatherUnroll; u++) {
            const uint32_t e = base + u * kGatherThreads;
            live[u] = e < total;
            if (live[u]) {
                const uint32_t row = fdiv(e, rv);
                const uint32_t col = e - row * rv.d;
                const int64_t id = __ldg(ids + row);
                const int4* src;
                if (placement) {
                    const uint64_t p = dev::ld_rand(placement + id);
                    const int b = (int)(p >> 40);
                    if (route && bins.owner[b] < 0 && (__ldg(route + row) % world) != self) {
                        live[u] = false;
                        continue;
                    }
                    src = bins.base[b] + (int64_t)(p & kSlotMask) * stride_vec + col;
                } else {
                    src = bins.base[0] + id * stride_vec + col;
                }
                val[u] = ld_stream(src);
            }
        }
#pragma unroll
        for (int u = 0; u < kGatherUnroll; u++)
            if (live[u]) out[base + u * kGatherThreads] = val[u];
    }
}

// ---- TMA bulk-copy gather (H6, local rows) ---------------------------------------------------------
// One warp per block. A tile is 32 consecutive output rows: lane l issues one cp.async.bulk global->smem
// copy of row l (completion counted in bytes on the stage's mbarrier); once the tile has landed, lane 0
// stores the whole tile (contiguous in the output) with ONE cp.async.bulk smem->global copy. kStages
// tiles are in flight per block, so an SM keeps kStages x blocks x 32 rows of reads outstanding with a
// handful of instructions per row.
constexpr int kBulkMaxRows = 32;
constexpr int kBulkSmemMax = 200 * 1024;  // dynamic shared memory a bulk-gather block may request

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
// L2 policies for the bulk copies: the gathered batch streams through L2 (evict_first) so it does not
// push the sampler's working set (CSR of hot vertices, bitmaps, lidx) out between batches.
__device__ __forceinline__ uint64_t l2_policy(int kind) {
    uint64_t p;
    if (kind == 1) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    else if (kind == 2) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    else asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void bulk_load(void* dst_smem, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
            smem_u32(dst_smem)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
}
__device__ __forceinline__ void bulk_store(void* dst, const void* src_smem, uint32_t bytes, uint64_t pol) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst),
                 "r"(smem_u32(src_smem)), "r"(bytes), "l"(pol)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
// Before a block exits only its shared memory must no longer be read by its bulk stores; the writes
// themselves complete with the grid (as CUTLASS's TMA-store epilogue tail does), so the last tile's write
// latency is not added to every block.
__device__ __forceinline__ void bulk_wait_exit() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }

// Source address of output row i (a row of bin b at slot s, or of the replicated table at slot id).
__device__ __forceinline__ const char* row_src(const BinTable& bins, const uint64_t* placement, int64_t id,
                                               int64_t stride) {
    if (placement) {
        const uint64_t p = dev::ld_rand(placement + id);
        return reinterpret_cast<const char*>(bins.base[(int)(p >> 40)]) + (int64_t)(p & kSlotMask) * stride;
    }
    return reinterpret_cast<const char*>(bins.base[0]) + id * stride;
}

template <int kBulkStages>
__global__ void __launch_bounds__(32) gather_bulk_kernel(BinTable bins, const uint64_t* __restrict__ placement,
                                                         const int64_t* __restrict__ ids, const int64_t* n_dev,
                                                         int64_t max_n, uint32_t R, int64_t stride,
                                                         int rows_per_tile, int l2_load, int l2_store,
                                                         char* __restrict__ out) {
    extern __shared__ __align__(128) char stage[];  // kBulkStages * rows_per_tile * R
    __shared__ __align__(8) uint64_t full[kBulkStages];
    const int lane = threadIdx.x;
    const uint64_t pol_ld = l2_policy(l2_load), pol_st = l2_policy(l2_store);
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    const int64_t n_tiles = (n + rows_per_tile - 1) / rows_per_tile;
    if (lane == 0)
        for (int s = 0; s < kBulkStages; s++) mbar_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncwarp();
    const int64_t t0 = blockIdx.x, dt = gridDim.x;
    // the source row of this lane in `tile`, resolved ahead of time (id load, then the placement lookup):
    // neither dependent load sits on the issue path
    auto load_id = [&](int64_t tile) -> const char* {
        const int64_t r = tile * rows_per_tile + lane;
        return (tile < n_tiles && lane < rows_per_tile && r < n) ? row_src(bins, placement, __ldg(ids + r), stride)
                                                                 : nullptr;
    };
    auto issue = [&](int64_t tile, int s, const char* src) {
        const int64_t row0 = tile * rows_per_tile;
        const int rows = (int)min((int64_t)rows_per_tile, n - row0);
        if (lane == 0) mbar_expect_tx(&full[s], (uint32_t)rows * R);
        __syncwarp();
        if (lane < rows) bulk_load(stage + ((size_t)s * rows_per_tile + lane) * R, src, R, &full[s], pol_ld);
    };
    // prologue: all ids of the first kBulkStages tiles in flight together, then their placement words, then
    // fill the pipeline
    int64_t pid[kBulkStages];
#pragma unroll
    for (int s = 0; s < kBulkStages; s++) {
        const int64_t tile = t0 + s * dt, r = tile * rows_per_tile + lane;
        pid[s] = (tile < n_tiles && lane < rows_per_tile && r < n) ? __ldg(ids + r) : -1;
    }
    const char* pre[kBulkStages];
#pragma unroll
    for (int s = 0; s < kBulkStages; s++) pre[s] = pid[s] >= 0 ? row_src(bins, placement, pid[s], stride) : nullptr;
    int64_t next = t0;
#pragma unroll
    for (int s = 0; s < kBulkStages; s++, next += dt)
        if (next < n_tiles) issue(next, s, pre[s]);
    const char* next_id = load_id(next);
    // steady state: store the tile that landed, then refill the stage of the PREVIOUS tile, whose store
    // was issued one iteration ago (wait_group.read 1: every store but the newest has read its stage).
    int it = 0;
    for (int64_t tile = t0; tile < n_tiles; tile += dt, it++) {
        const int s = it % kBulkStages;
        mbar_wait(&full[s], (uint32_t)((it / kBulkStages) & 1));
        const int64_t row0 = tile * rows_per_tile;
        const int rows = (int)min((int64_t)rows_per_tile, n - row0);
        if (lane == 0) {
            bulk_store(out + row0 * (int64_t)R, stage + (size_t)s * rows_per_tile * R, (uint32_t)rows * R, pol_st);
            if (it > 0) bulk_wait_read<1>();
        }
        __syncwarp();
        if (it > 0 && next < n_tiles) {
            issue(next, (it - 1) % kBulkStages, next_id);
            next += dt;
            next_id = load_id(next);
        }
    }
    if (lane == 0) bulk_wait_exit();
}

// TMA tile::gather4 variant of the bulk gather (sm_100a): one tensor copy fetches FOUR rows of the
// replicated table (a 2-D tensor map over [n rows][R / 4 words] with the table's row stride), so a
// 32-row tile is 8 copies instead of 32. The tensor map also carries the L2 promotion (fetch) size of the
// reads. Each group of 4 rows lands at a 128-byte aligned smem slot (G bytes) and is stored back with its
// own bulk copy (per-lane bulk groups). Rows past the end of a tile repeat the tile's first row and are
// not stored.
constexpr int kTma4Rows = 32;  // rows per tile = 8 groups of 4 (kRows = 16 / 8: 4 / 2 groups; ctx tma4_rows)
template <int kStages, bool kPlacement, int kRows = kTma4Rows>
__global__ void __launch_bounds__(32) gather_tma4_kernel(const __grid_constant__ CUtensorMap tmap,
                                                         const int64_t* __restrict__ ids, const int64_t* n_dev,
                                                         int64_t max_n, uint32_t R, int l2_load, int l2_store,
                                                         const uint64_t* __restrict__ placement,
                                                         char* __restrict__ out) {
    extern __shared__ __align__(128) char stage[];  // kStages * 8 * G
    __shared__ __align__(8) uint64_t full[kStages];
    const int lane = threadIdx.x;
    const uint32_t G = (4 * R + 127) & ~127u;
    const uint64_t pol_st = l2_policy(l2_store), pol_ld = l2_policy(l2_load);
    const int64_t t0 = blockIdx.x, dt = gridDim.x;
    if (lane == 0) asm volatile("prefetch.tensormap [%0];" ::"l"(&tmap) : "memory");
    // the first kStages tiles' ids are loaded speculatively (bounded by max_n, the ids buffer) together with
    // the count instead of after it: one dependent global round trip fewer before the first row request.
    // Ids past the count are never used (issue() replaces them by the tile's first row).
    int32_t pre[kStages];
    int64_t pid[kStages];
#pragma unroll
    for (int s = 0; s < kStages; s++) {
        const int64_t r = (t0 + s * dt) * kRows + lane;
        // lanes past the tile's rows: their loads (the next tile's ids) act as a prefetch in the replicated
        // instantiation (single launch 0.70 -> 0.71 with them); behind a placement map they would add a random
        // lookup per row, so there they load nothing
        pid[s] = ((!kPlacement || lane < kRows) && r < max_n) ? __ldg(ids + r) : -1;
    }
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    // kPlacement (one local bin behind a placement map, e.g. a DDAK layout on one GPU): the row coordinate is
    // the slot, one more dependent load after the id (its own instantiation: the replicated path keeps the
    // count load in flight together with the first ids)
    // (ids past the count are stale buffer contents: never looked up)
#pragma unroll
    for (int s = 0; s < kStages; s++)
        pre[s] = !kPlacement ? (int32_t)pid[s]
                 : (lane < kRows && (t0 + s * dt) * kRows + lane < n ? (int32_t)(dev::ld_rand(placement + pid[s]) & kSlotMask) : -1);
    const int64_t n_tiles = (n + kRows - 1) / kRows;
    if (lane == 0)
        for (int s = 0; s < kStages; s++) mbar_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncwarp();
    auto load_id = [&](int64_t tile) -> int32_t {
        const int64_t r = tile * kRows + lane;
        if (!((!kPlacement || lane < kRows) && tile < n_tiles && r < n)) return -1;
        const int64_t id = __ldg(ids + r);
        return kPlacement ? (int32_t)(dev::ld_rand(placement + id) & kSlotMask) : (int32_t)id;
    };
    auto issue = [&](int64_t tile, int s, int32_t id) {
        const int rows = (int)min((int64_t)kRows, n - tile * kRows);
        const int groups = (rows + 3) >> 2;
        const int32_t first = __shfl_sync(0xffffffffu, id, 0);
        const int32_t rid = lane < rows ? id : first;
        const int g = lane & (kRows / 4 - 1);
        const int32_t r0 = __shfl_sync(0xffffffffu, rid, 4 * g), r1 = __shfl_sync(0xffffffffu, rid, 4 * g + 1);
        const int32_t r2 = __shfl_sync(0xffffffffu, rid, 4 * g + 2), r3 = __shfl_sync(0xffffffffu, rid, 4 * g + 3);
        if (lane == 0) mbar_expect_tx(&full[s], (uint32_t)groups * 4u * R);
        __syncwarp();
        if (lane < groups) {
            if (l2_load)  // L2 eviction priority of the fetched rows (MOMENT_GATHER_L2 first digit)
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes.L2::cache_hint "
                    "[%0], [%1, {%2, %3, %4, %5, %6}], [%7], %8;" ::"r"(smem_u32(stage + ((size_t)s * (kRows / 4) + lane) * G)),
                    "l"(&tmap), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(smem_u32(&full[s])), "l"(pol_ld)
                    : "memory");
            else
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, "
                    "%3, %4, %5, %6}], [%7];" ::"r"(smem_u32(stage + ((size_t)s * (kRows / 4) + lane) * G)),
                    "l"(&tmap), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(smem_u32(&full[s]))
                    : "memory");
        }
    };
    int64_t next = t0;
#pragma unroll
    for (int s = 0; s < kStages; s++, next += dt)
        if (next < n_tiles) issue(next, s, pre[s]);
    int32_t next_id = load_id(next);
    int it = 0;
    for (int64_t tile = t0; tile < n_tiles; tile += dt, it++) {
        const int s = it % kStages;
        mbar_wait(&full[s], (uint32_t)((it / kStages) & 1));
        const int64_t row0 = tile * kRows;
        const int rows = (int)min((int64_t)kRows, n - row0);
        const int groups = (rows + 3) >> 2;
        if (lane < groups) {
            bulk_store(out + (row0 + 4 * lane) * (int64_t)R, stage + ((size_t)s * (kRows / 4) + lane) * G,
                       (uint32_t)min(4, rows - 4 * lane) * R, pol_st);
        }
        if (it > 0) bulk_wait_read<1>();  // this lane's store of the previous tile has read its slot
        __syncwarp();
        if (it > 0 && next < n_tiles) {
            issue(next, (it - 1) % kStages, next_id);
            next += dt;
            next_id = load_id(next);
            {  // the ids one more tile ahead into L2 (single launch 0.72 -> 0.73 of the copy peak)
                const int64_t r2 = (next + dt) * kRows + lane;
                if (lane < kRows && next + dt < n_tiles && r2 < n) asm volatile("prefetch.global.L2 [%0];" ::"l"(ids + r2));
            }
        }
    }
    bulk_wait_exit();
}

// Relay service (H7): this rank (server) reads the host rows that `requester` routed through it and
// stores them into the requester's output (an NVLink store when the requester is another GPU).
// Requests are the queue segments q = j * world + server of every host bin j.
__global__ void __launch_bounds__(kGatherThreads) relay_kernel(BinTable bins, const uint64_t* __restrict__ placement,
                                                               const int64_t* __restrict__ ids,
                                                               const int64_t* __restrict__ qoff,
                                                               const int64_t* __restrict__ qpos, int32_t n_bins,
                                                               int32_t world, int32_t server, FastDiv rv,
                                                               int64_t stride_vec, int4* __restrict__ out) {
    for (int b = 0; b < n_bins; b++) {
        if (bins.owner[b] >= 0) continue;  // HBM bins are read by the requester itself (peer load)
        const int q = b * world + server;
        const int64_t lo = qoff[q], cnt = qoff[q + 1] - lo;
        const uint32_t total = (uint32_t)(cnt * rv.d);
        for (uint32_t e = blockIdx.x * kGatherThreads + threadIdx.x; e < total; e += gridDim.x * kGatherThreads) {
            const uint32_t r = fdiv(e, rv);
            const uint32_t col = e - r * rv.d;
            const int64_t i = __ldg(qpos + lo + r);
            const uint64_t p = __ldg(placement + __ldg(ids + i));
            const int4 v = ld_stream(bins.base[(int)(p >> 40)] + (int64_t)(p & kSlotMask) * stride_vec + col);
            out[i * rv.d + col] = v;
        }
    }
}

// ---- bucketing (H4) -------------------------------------------------------------------------------
// Pass 1: per tile of kBucketTile requests, per-bin counts.
__global__ void bucket_count_kernel(const uint64_t* __restrict__ placement, const int64_t* __restrict__ ids,
                                    const int64_t* n_dev, int64_t max_n, int32_t n_bins, int64_t* tile_counts) {
    __shared__ int s_cnt[MOMENT_MAX_BINS];
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    const int64_t n_tiles_max = (max_n + kBucketTile - 1) / kBucketTile;
    for (int64_t tile = blockIdx.x; tile < n_tiles_max; tile += gridDim.x) {
        for (int b = threadIdx.x; b < n_bins; b += blockDim.x) s_cnt[b] = 0;
        __syncthreads();
        for (int64_t i = tile * kBucketTile + threadIdx.x; i < min(n, (tile + 1) * kBucketTile); i += blockDim.x) {
            const int b = (int)(__ldg(placement + __ldg(ids + i)) >> 40);
            atomicAdd(&s_cnt[b], 1);
        }
        __syncthreads();
        for (int b = threadIdx.x; b < n_bins; b += blockDim.x) tile_counts[tile * n_bins + b] = s_cnt[b];
        __syncthreads();
    }
}

// Pass 2 (one block): exclusive scan over tiles per bin; bin totals.
__global__ void bucket_scan_kernel(int64_t* tile_counts, int64_t n_tiles, int32_t n_bins, int64_t* bin_total) {
    for (int b = threadIdx.x; b < n_bins; b += blockDim.x) {
        int64_t run = 0;
        for (int64_t t = 0; t < n_tiles; t++) {
            const int64_t c = tile_counts[t * n_bins + b];
            tile_counts[t * n_bins + b] = run;
            run += c;
        }
        bin_total[b] = run;
    }
}

// Pass 3: stable rank r of each request inside its bin -> route. A host bin j with W = sum_h x[j][h]
// sends rank r through the first h with floor(r W / n_j) < cumsum_h x[j][.]; equivalently rank r goes
// to h iff r_lo(h) <= r < r_lo(h+1), r_lo(h) = ceil(C_h n_j / W), C_h = sum_{h'<h} x[j][h'].
__global__ void __launch_bounds__(kBucketTile) bucket_route_kernel(
    const uint64_t* __restrict__ placement, const int64_t* __restrict__ ids, const int64_t* n_dev, int64_t max_n,
    int32_t n_bins, int32_t world, int32_t self, const int32_t* __restrict__ bin_owner_dev,
    const int64_t* __restrict__ quota, const int64_t* __restrict__ tile_base, const int64_t* __restrict__ bin_total,
    int32_t* __restrict__ route) {
    __shared__ int s_warp_cnt[kBucketTile / 32][MOMENT_MAX_BINS];
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    const int64_t n_tiles_max = (max_n + kBucketTile - 1) / kBucketTile;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int64_t tile = blockIdx.x; tile < n_tiles_max; tile += gridDim.x) {
        const int64_t i = tile * kBucketTile + threadIdx.x;
        const bool live = i < n;
        const int b = live ? (int)(__ldg(placement + __ldg(ids + i)) >> 40) : -1;
        // rank within the warp among equal bins, then within the tile via per-warp counts
        const unsigned peers = __match_any_sync(0xffffffffu, b);
        const int in_warp = __popc(peers & ((1u << lane) - 1));
        for (int q = lane; q < n_bins; q += 32) s_warp_cnt[wid][q] = 0;
        __syncwarp();
        if (live && in_warp == 0) s_warp_cnt[wid][b] = __popc(peers);
        __syncthreads();
        if (live) {
            int before = 0;
            for (int w = 0; w < wid; w++) before += s_warp_cnt[w][b];
            const int64_t r = tile_base[tile * n_bins + b] + before + in_warp;
            int via;
            const int owner = bin_owner_dev[b];
            if (owner >= 0) {
                via = owner;
            } else {
                const int64_t* x = quota + (int64_t)b * world;
                int64_t W = 0;
                for (int h = 0; h < world; h++) W += x[h];
                if (W == 0) {
                    via = self;
                } else {
                    const int64_t nj = bin_total[b];
                    // slot = floor(r W / nj) (int128), via = first h with slot < cumsum
                    const unsigned __int128 prod = (unsigned __int128)r * (unsigned __int128)W;
                    const int64_t slot = (int64_t)(prod / (unsigned __int128)nj);
                    int64_t cum = 0;
                    via = world - 1;
                    for (int h = 0; h < world; h++) {
                        cum += x[h];
                        if (slot < cum) { via = h; break; }
                    }
                }
            }
            route[i] = b * world + via;
        }
        __syncthreads();
    }
}

// Queue layout: stable counting sort of requests by route (q = bin * world + via).
__global__ void queue_count_kernel(const int32_t* __restrict__ route, const int64_t* n_dev, int64_t max_n, int32_t Q,
                                   int64_t* tile_counts) {
    __shared__ int s_cnt[kMaxQueues];
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    const int64_t n_tiles_max = (max_n + kBucketTile - 1) / kBucketTile;
    for (int64_t tile = blockIdx.x; tile < n_tiles_max; tile += gridDim.x) {
        for (int q = threadIdx.x; q < Q; q += blockDim.x) s_cnt[q] = 0;
        __syncthreads();
        for (int64_t i = tile * kBucketTile + threadIdx.x; i < min(n, (tile + 1) * kBucketTile); i += blockDim.x)
            atomicAdd(&s_cnt[route[i]], 1);
        __syncthreads();
        for (int q = threadIdx.x; q < Q; q += blockDim.x) tile_counts[tile * Q + q] = s_cnt[q];
        __syncthreads();
    }
}

// One block: qoff[q] = sum of all counts of queues < q; tile_counts -> absolute tile bases.
__global__ void queue_scan_kernel(int64_t* tile_counts, int64_t n_tiles, int32_t Q, int64_t* qoff) {
    __shared__ int64_t s_tot[kMaxQueues + 1];
    for (int q = threadIdx.x; q < Q; q += blockDim.x) {
        int64_t run = 0;
        for (int64_t t = 0; t < n_tiles; t++) {
            const int64_t c = tile_counts[t * Q + q];
            tile_counts[t * Q + q] = run;
            run += c;
        }
        s_tot[q] = run;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        int64_t run = 0;
        for (int q = 0; q < Q; q++) {
            qoff[q] = run;
            run += s_tot[q];
        }
        qoff[Q] = run;
    }
    __syncthreads();
    for (int q = threadIdx.x; q < Q; q += blockDim.x)
        for (int64_t t = 0; t < n_tiles; t++) tile_counts[t * Q + q] += qoff[q];
}

__global__ void __launch_bounds__(kBucketTile) queue_scatter_kernel(const int32_t* __restrict__ route,
                                                                    const int64_t* n_dev, int64_t max_n, int32_t Q,
                                                                    const int64_t* __restrict__ tile_base,
                                                                    int64_t* __restrict__ qpos) {
    __shared__ int s_warp_cnt[kBucketTile / 32][kMaxQueues];
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    const int64_t n_tiles_max = (max_n + kBucketTile - 1) / kBucketTile;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int64_t tile = blockIdx.x; tile < n_tiles_max; tile += gridDim.x) {
        const int64_t i = tile * kBucketTile + threadIdx.x;
        const bool live = i < n;
        const int q = live ? route[i] : -1;
        const unsigned peers = __match_any_sync(0xffffffffu, q);
        const int in_warp = __popc(peers & ((1u << lane) - 1));
        for (int c = lane; c < Q; c += 32) s_warp_cnt[wid][c] = 0;
        __syncwarp();
        if (live && in_warp == 0) s_warp_cnt[wid][q] = __popc(peers);
        __syncthreads();
        if (live) {
            int before = 0;
            for (int w = 0; w < wid; w++) before += s_warp_cnt[w][q];
            qpos[tile_base[tile * Q + q] + before + in_warp] = i;
        }
        __syncthreads();
    }
}

__global__ void hotness_kernel(const int64_t* __restrict__ ids, const int64_t* n_dev, int64_t max_n, uint64_t* hot) {
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(reinterpret_cast<unsigned long long*>(hot + __ldg(ids + i)), 1ull);
}

BinTable make_bins(const moment_ctx_s* ctx) {
    BinTable t{};
    for (int b = 0; b < ctx->n_bins; b++) {
        t.base[b] = reinterpret_cast<const int4*>(ctx->bin_ptr[b]);
        t.owner[b] = (int8_t)ctx->bin_owner[b];
    }
    return t;
}

int grid_for(int64_t work_items, int per_block, int max_blocks) {
    return (int)std::max<int64_t>(1, std::min<int64_t>((work_items + per_block - 1) / per_block, max_blocks));
}

// Tensor map of the replicated table for tile::gather4: 2-D, 32-bit elements, [n_vertices][R / 4] with the
// table's row stride, box = one row; built once per table pointer (cuTensorMapEncodeTiled is resolved
// from the driver at run time, so the library does not link libcuda).
moment_status encode_table_map(moment_ctx_s* ctx) {
    using encode_fn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
    static encode_fn encode = nullptr;
    if (!encode) {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        MOMENT_TRY(cuda_check(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q),
                              "moment_gather: driver entry point"));
        if (!fn || q != cudaDriverEntryPointSuccess) return fail(MOMENT_ECUDA, "moment_gather: cuTensorMapEncodeTiled missing");
        encode = reinterpret_cast<encode_fn>(fn);
    }
    const cuuint64_t dims[2] = {(cuuint64_t)(ctx->row_bytes / 4), (cuuint64_t)ctx->n_vertices};
    const cuuint64_t strides[1] = {(cuuint64_t)ctx->row_stride};
    const cuuint32_t box[2] = {(cuuint32_t)(ctx->row_bytes / 4), 1};
    const cuuint32_t estr[2] = {1, 1};
    const CUresult r = encode(&ctx->tma_map, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, ctx->bin_ptr[0], dims, strides, box, estr,
                              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                              (CUtensorMapL2promotion)ctx->tma_promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return fail(MOMENT_ECUDA, "moment_gather: cuTensorMapEncodeTiled failed (%d)", (int)r);
    ctx->tma_base = ctx->bin_ptr[0];
    return MOMENT_OK;
}

}  // namespace

moment_status launch_gather(moment_ctx_s* ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n, void* out,
                            const int32_t* route, int32_t serve_rank, cudaStream_t stream) {
    if (max_n < 0 || (max_n > 0 && (!ids || !out))) return fail(MOMENT_EINVAL, "moment_gather: null argument");
    if (ctx->n_bins <= 0) return fail(MOMENT_EINVAL, "moment_gather: ctx has no feature bins");
    const int64_t rv = ctx->row_bytes / 16;
    if (max_n * rv >= (int64_t(1) << 32))
        return fail(MOMENT_EUNSUPPORTED, "moment_gather: %lld rows x %lld vectors exceeds 2^32 per call", (long long)max_n, (long long)rv);
    if ((reinterpret_cast<uintptr_t>(out) & 15) != 0) return fail(MOMENT_EINVAL, "moment_gather: out must be 16-byte aligned");
    MOMENT_TRY(cuda_pending("moment_gather: pending CUDA error"));
    if (max_n == 0) return MOMENT_OK;
    bool all_local = true;
    for (int b = 0; b < ctx->n_bins; b++) all_local &= ctx->bin_owner[b] == ctx->rank;
    // auto: tile::gather4 for a replicated table whose row fits one box (<= 256 words), TMA bulk copies for
    // other local rows, LDG.128 for routed / remote rows
    // (a placement map with one local bin, e.g. DDAK on one GPU: the coordinate is the slot, < 2^31 rows)
    const bool tma4_ok = route == nullptr && ctx->n_bins == 1 && all_local && ctx->row_bytes / 4 <= 256 &&
                         ctx->n_vertices < (int64_t(1) << 31);
    const bool tma4 = tma4_ok && (ctx->gather_path == 3 || ctx->gather_path == 0);
    const bool bulk = ctx->gather_path == 2 || (ctx->gather_path == 0 && route == nullptr && all_local);
    if (tma4) {
        if (ctx->tma_base != ctx->bin_ptr[0]) MOMENT_TRY(encode_table_map(ctx));
        const uint32_t G = (uint32_t)((4 * ctx->row_bytes + 127) & ~int64_t(127));
        // launch shape (ctx.h): 16-row tiles x 3 blocks/SM for both instantiations (behind a placement map, C3 DDAK:
        // 32 x 2 streams a lone launch at 0.62 instead of 0.57 but the bench runs 1.5 % slower)
        const int stages = 4, bps = ctx->tma4_blocks_per_sm;
        const int rows_t = ctx->tma4_rows <= 8 ? 8 : ctx->tma4_rows <= 16 ? 16 : 32;
        const size_t smem = (size_t)stages * (rows_t / 4) * G;
        const int64_t tiles = (max_n + rows_t - 1) / rows_t;
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, (int64_t)device_sms() * bps));
        auto launch = [&](auto kern) {
            kern<<<grid, 32, smem, stream>>>(ctx->tma_map, ids, n_dev, max_n, (uint32_t)ctx->row_bytes, ctx->l2_load_policy,
                                             ctx->l2_store_policy, ctx->placement, reinterpret_cast<char*>(out));
        };
        if (ctx->placement) {
            if (rows_t == 8) launch(gather_tma4_kernel<4, true, 8>);
            else if (rows_t == 16) launch(gather_tma4_kernel<4, true, 16>);
            else launch(gather_tma4_kernel<4, true>);
        } else {
            if (rows_t == 8) launch(gather_tma4_kernel<4, false, 8>);
            else if (rows_t == 16) launch(gather_tma4_kernel<4, false, 16>);
            else launch(gather_tma4_kernel<4, false>);
        }
        return cuda_check(cudaGetLastError(), "moment_gather: tma4 launch");
    }
    if (bulk && route == nullptr) {
        // tiles of <= 32 rows, `stages` tiles in flight per 1-warp block, `bps` blocks per SM, each stage at
        // most `stage_kb` KB (defaults 4 / 4 / 14: 4 x 4 x 14 KB fits the SM's shared memory)
        const int bps = ctx->bulk_blocks_per_sm;  // stages rounded up to an instantiated pipeline depth
        const int stages = ctx->bulk_stages <= 2 ? 2 : ctx->bulk_stages <= 4 ? 4 : ctx->bulk_stages <= 6 ? 6 : 8;
        const int rows = (int)std::max<int64_t>(1, std::min<int64_t>(kBulkMaxRows, ctx->bulk_stage_kb * 1024 / ctx->row_bytes));
        const size_t smem = (size_t)stages * rows * ctx->row_bytes;
        if (smem > (size_t)kBulkSmemMax) return fail(MOMENT_EINVAL, "moment_gather: bulk stage config needs %zu B smem", smem);
        const int64_t tiles = (max_n + rows - 1) / rows;
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, (int64_t)device_sms() * bps));
        auto launch = [&](auto kern) {
            kern<<<grid, 32, smem, stream>>>(make_bins(ctx), ctx->placement, ids, n_dev, max_n, (uint32_t)ctx->row_bytes,
                                             ctx->row_stride, rows, ctx->l2_load_policy, ctx->l2_store_policy,
                                             reinterpret_cast<char*>(out));
        };
        if (stages <= 2) launch(gather_bulk_kernel<2>);
        else if (stages <= 4) launch(gather_bulk_kernel<4>);
        else if (stages <= 6) launch(gather_bulk_kernel<6>);
        else launch(gather_bulk_kernel<8>);
    } else {
        const int grid = grid_for(max_n * rv, kGatherThreads * kGatherUnroll, device_sms() * 8);
        gather_kernel<<<grid, kGatherThreads, 0, stream>>>(make_bins(ctx), ctx->placement, ids, n_dev, max_n,
                                                            make_fastdiv((uint32_t)rv), ctx->row_stride / 16, route,
                                                            ctx->world, serve_rank, reinterpret_cast<int4*>(out));
    }
    return cuda_check(cudaGetLastError(), "moment_gather: launch");
}

moment_status launch_bucket(moment_ctx_s* ctx, const int64_t* ids, const int64_t* n_dev, int64_t max_n,
                            int32_t* route, int64_t* qoff, int64_t* qpos, cudaStream_t stream) {
    if (!ctx->placement) return fail(MOMENT_EINVAL, "moment_bucket: ctx has no placement map");
    if (max_n > ctx->max_requests)
        return fail(MOMENT_EOVERFLOW, "moment_bucket: %lld requests > workspace %lld", (long long)max_n, (long long)ctx->max_requests);
    const int32_t Q = ctx->n_bins * ctx->world;
    if (Q > kMaxQueues) return fail(MOMENT_EUNSUPPORTED, "moment_bucket: n_bins * world = %d > %d", Q, kMaxQueues);
    MOMENT_TRY(cuda_pending("moment_bucket: pending CUDA error"));
    if (max_n == 0)  // no requests: empty queues (the tile kernels below would read stale tile counts)
        return cuda_check(cudaMemsetAsync(qoff, 0, (size_t)(Q + 1) * sizeof(int64_t), stream), "moment_bucket: empty");
    const int64_t n_tiles = std::max<int64_t>(1, (max_n + kBucketTile - 1) / kBucketTile);
    const int grid = (int)std::min<int64_t>(n_tiles, device_sms() * 2);
    bucket_count_kernel<<<grid, 256, 0, stream>>>(ctx->placement, ids, n_dev, max_n, ctx->n_bins, ctx->bk_tile_counts);
    bucket_scan_kernel<<<1, 64, 0, stream>>>(ctx->bk_tile_counts, n_tiles, ctx->n_bins, ctx->bk_bin_total);
    const int32_t* owner_dev = ctx->d_bin_owner;
    bucket_route_kernel<<<grid, kBucketTile, 0, stream>>>(ctx->placement, ids, n_dev, max_n, ctx->n_bins, ctx->world,
                                                          ctx->rank, owner_dev, ctx->d_quota, ctx->bk_tile_counts,
                                                          ctx->bk_bin_total, route);
    queue_count_kernel<<<grid, 256, 0, stream>>>(route, n_dev, max_n, Q, ctx->bk_tile_counts);
    queue_scan_kernel<<<1, 256, 0, stream>>>(ctx->bk_tile_counts, n_tiles, Q, qoff);
    queue_scatter_kernel<<<grid, kBucketTile, 0, stream>>>(route, n_dev, max_n, Q, ctx->bk_tile_counts, qpos);
    return cuda_check(cudaGetLastError(), "moment_bucket: launch");
}

moment_status launch_relay(moment_ctx_s* server, moment_ctx_s* requester, const int64_t* ids, const int32_t* route,
                           const int64_t* qoff, const int64_t* qpos, void* requester_out, cudaStream_t stream) {
    (void)route;
    const int64_t rv = server->row_bytes / 16;
    const int grid = device_sms() * 4;
    relay_kernel<<<grid, kGatherThreads, 0, stream>>>(make_bins(server), requester->placement, ids, qoff, qpos,
                                                       server->n_bins, server->world, server->rank,
                                                       make_fastdiv((uint32_t)rv), server->row_stride / 16,
                                                       reinterpret_cast<int4*>(requester_out));
    return cuda_check(cudaGetLastError(), "moment_gather: relay launch");
}

// ---- H5 exchange for one process per GPU (all-to-all transport) ---------------------------------------
namespace {

constexpr int kMaxSegs = 128;  // (destination rank, host bin) segments

// Segments of this rank's relay queues in send order (destination h ascending, then host bin b):
// q = b * world + h for h != self and host bins b. Computed redundantly by every block (<= 128 entries).
__device__ int build_segments(const int64_t* qoff, const BinTable& bins, int n_bins, int world, int self,
                              int64_t* seg_src, int64_t* seg_dst, int* seg_h) {
    int n = 0;
    int64_t dst = 0;
    for (int h = 0; h < world; h++) {
        if (h == self) continue;
        for (int b = 0; b < n_bins; b++) {
            if (bins.owner[b] >= 0) continue;
            const int q = b * world + h;
            seg_src[n] = qoff[q];
            seg_dst[n] = dst;
            seg_h[n] = h;
            dst += qoff[q + 1] - qoff[q];
            n++;
        }
    }
    seg_dst[n] = dst;
    return n;
}

// words[2e] = placement word of the row, words[2e+1] = its position in this rank's output; counts[h] =
// entries for destination h (0 for self).
__global__ void relay_pack_kernel(BinTable bins, const uint64_t* __restrict__ placement, const int64_t* __restrict__ ids,
                                  const int64_t* __restrict__ qoff, const int64_t* __restrict__ qpos, int32_t n_bins,
                                  int32_t world, int32_t self, uint64_t* __restrict__ words, int64_t* counts) {
    __shared__ int64_t s_src[kMaxSegs + 1], s_dst[kMaxSegs + 1];
    __shared__ int s_h[kMaxSegs + 1];
    __shared__ int s_n;
    if (threadIdx.x == 0) s_n = build_segments(qoff, bins, n_bins, world, self, s_src, s_dst, s_h);
    __syncthreads();
    const int ns = s_n;
    if (blockIdx.x == 0 && threadIdx.x < world) {
        int64_t c = 0;
        for (int s = 0; s < ns; s++)
            if (s_h[s] == (int)threadIdx.x) c += s_dst[s + 1] - s_dst[s];
        counts[threadIdx.x] = c;
    }
    const int64_t total = s_dst[ns];
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        int lo = 0, hi = ns - 1;
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (s_dst[mid] <= e) lo = mid;
            else hi = mid - 1;
        }
        const int64_t i = __ldg(qpos + s_src[lo] + (e - s_dst[lo]));
        words[2 * e] = __ldg(placement + __ldg(ids + i));
        words[2 * e + 1] = (uint64_t)i;
    }
}

// rows[e] = the row named by placement word words[2e], read by THIS rank (its host-bin mapping).
__global__ void __launch_bounds__(kGatherThreads) relay_serve_kernel(BinTable bins, const uint64_t* __restrict__ words,
                                                                     const int64_t* n_dev, int64_t max_n, FastDiv rv,
                                                                     int64_t stride_vec, int4* __restrict__ rows) {
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    const uint32_t total = (uint32_t)(n * rv.d);
    for (uint32_t v = blockIdx.x * kGatherThreads + threadIdx.x; v < total; v += gridDim.x * kGatherThreads) {
        const uint32_t e = fdiv(v, rv), col = v - e * rv.d;
        const uint64_t p = __ldg(words + 2 * (int64_t)e);
        rows[v] = ld_stream(bins.base[(int)(p >> 40)] + (int64_t)(p & kSlotMask) * stride_vec + col);
    }
}

// out[words[2e+1]] = rows[e].
__global__ void __launch_bounds__(kGatherThreads) relay_scatter_kernel(const uint64_t* __restrict__ words,
                                                                       const int64_t* n_dev, int64_t max_n, FastDiv rv,
                                                                       const int4* __restrict__ rows,
                                                                       int4* __restrict__ out) {
    const int64_t n = n_dev ? min(*n_dev, max_n) : max_n;
    const uint32_t total = (uint32_t)(n * rv.d);
    for (uint32_t v = blockIdx.x * kGatherThreads + threadIdx.x; v < total; v += gridDim.x * kGatherThreads) {
        const uint32_t e = fdiv(v, rv), col = v - e * rv.d;
        out[(int64_t)__ldg(words + 2 * (int64_t)e + 1) * rv.d + col] = ld_stream(rows + v);
    }
}

// ---- the same exchange over peer memory (no all-to-all) ------------------------------------------------
struct PeerInboxes {
    uint64_t* inbox[MOMENT_MAX_WORLD];  // rank h's inbox slot for this rank (peer pointer)
    int64_t* count[MOMENT_MAX_WORLD];   // rank h's count slot for this rank (peer pointer)
};
struct PeerOuts {
    int4* out[MOMENT_MAX_WORLD];  // rank g's batch output (peer pointer)
};

// relay_pack with the words stored straight into the destination rank's inbox: one 16-byte peer store per
// request (placement word, output position), and the per-destination count into the peer's count slot.
__global__ void relay_push_kernel(BinTable bins, const uint64_t* __restrict__ placement, const int64_t* __restrict__ ids,
                                  const int64_t* __restrict__ qoff, const int64_t* __restrict__ qpos, int32_t n_bins,
                                  int32_t world, int32_t self, PeerInboxes peers) {
    __shared__ int64_t s_src[kMaxSegs + 1], s_dst[kMaxSegs + 1], s_hbase[MOMENT_MAX_WORLD];
    __shared__ int s_h[kMaxSegs + 1];
    __shared__ int s_n;
    if (threadIdx.x == 0) {
        s_n = build_segments(qoff, bins, n_bins, world, self, s_src, s_dst, s_h);
        for (int h = 0; h < world; h++) s_hbase[h] = -1;
        for (int s = s_n - 1; s >= 0; s--) s_hbase[s_h[s]] = s_dst[s];  // first word of destination h
    }
    __syncthreads();
    const int ns = s_n;
    if (blockIdx.x == 0 && threadIdx.x < world && (int)threadIdx.x != self) {
        int64_t c = 0;
        for (int s = 0; s < ns; s++)
            if (s_h[s] == (int)threadIdx.x) c += s_dst[s + 1] - s_dst[s];
        *peers.count[threadIdx.x] = c;
    }
    const int64_t total = s_dst[ns];
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        int lo = 0, hi = ns - 1;
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (s_dst[mid] <= e) lo = mid;
            else hi = mid - 1;
        }
        const int h = s_h[lo];
        const int64_t i = __ldg(qpos + s_src[lo] + (e - s_dst[lo]));
        const ulonglong2 w = make_ulonglong2(__ldg(placement + __ldg(ids + i)), (unsigned long long)i);
        reinterpret_cast<ulonglong2*>(peers.inbox[h])[e - s_hbase[h]] = w;
    }
}

// Serve every source rank's inbox: read the host row named by each request from THIS rank's mapping of
// the host bins and store it straight into the source's output row (peer stores).
__global__ void __launch_bounds__(kGatherThreads) relay_serve_push_kernel(BinTable bins, const uint64_t* __restrict__ inbox,
                                                                          const int64_t* __restrict__ inbox_count,
                                                                          int64_t cap, int32_t world, int32_t self,
                                                                          FastDiv rv, int64_t stride_vec, PeerOuts outs) {
    __shared__ int64_t s_off[MOMENT_MAX_WORLD + 1];
    if (threadIdx.x == 0) {
        int64_t o = 0;
        for (int g = 0; g < world; g++) {
            s_off[g] = o;
            o += g == self ? 0 : min(max(inbox_count[g], (int64_t)0), cap);
        }
        s_off[world] = o;
    }
    __syncthreads();
    const int64_t total = s_off[world] * rv.d;
    for (int64_t v = (int64_t)blockIdx.x * kGatherThreads + threadIdx.x; v < total; v += (int64_t)gridDim.x * kGatherThreads) {
        const int64_t e = v / rv.d;
        const int col = (int)(v - e * rv.d);
        int g = 0;
        while (s_off[g + 1] <= e) g++;
        const int64_t r = e - s_off[g];
        const uint64_t* w = inbox + 2 * ((int64_t)g * cap + r);
        const uint64_t p = __ldg(w), pos = __ldg(w + 1);
        outs.out[g][(int64_t)pos * rv.d + col] =
            ld_stream(bins.base[(int)(p >> 40)] + (int64_t)(p & kSlotMask) * stride_vec + col);
    }
}

}  // namespace

moment_status launch_relay_pack(moment_ctx_s* ctx, const int64_t* ids, const int64_t* qoff, const int64_t* qpos,
                                int64_t max_n, uint64_t* words, int64_t* counts, cudaStream_t stream) {
    if (!ctx->placement) return fail(MOMENT_EINVAL, "moment_relay_pack: ctx has no placement map");
    if (ctx->n_bins * (ctx->world - 1) > kMaxSegs) return fail(MOMENT_EUNSUPPORTED, "moment_relay_pack: too many segments");
    const int grid = grid_for(std::max<int64_t>(max_n, 1), 256, device_sms() * 4);
    relay_pack_kernel<<<grid, 256, 0, stream>>>(make_bins(ctx), ctx->placement, ids, qoff, qpos, ctx->n_bins, ctx->world,
                                                ctx->rank, words, counts);
    return cuda_check(cudaGetLastError(), "moment_relay_pack: launch");
}

moment_status launch_relay_serve(moment_ctx_s* ctx, const uint64_t* words, const int64_t* n_dev, int64_t max_n,
                                 void* rows, cudaStream_t stream) {
    const int64_t rv = ctx->row_bytes / 16;
    if (max_n * rv >= (int64_t(1) << 32)) return fail(MOMENT_EUNSUPPORTED, "moment_relay_serve: too many rows");
    if (max_n == 0) return MOMENT_OK;
    relay_serve_kernel<<<grid_for(max_n * rv, kGatherThreads, device_sms() * 8), kGatherThreads, 0, stream>>>(
        make_bins(ctx), words, n_dev, max_n, make_fastdiv((uint32_t)rv), ctx->row_stride / 16,
        reinterpret_cast<int4*>(rows));
    return cuda_check(cudaGetLastError(), "moment_relay_serve: launch");
}

moment_status launch_relay_scatter(moment_ctx_s* ctx, const uint64_t* words, const int64_t* n_dev, int64_t max_n,
                                   const void* rows, void* out, cudaStream_t stream) {
    const int64_t rv = ctx->row_bytes / 16;
    if (max_n * rv >= (int64_t(1) << 32)) return fail(MOMENT_EUNSUPPORTED, "moment_relay_scatter: too many rows");
    if (max_n == 0) return MOMENT_OK;
    relay_scatter_kernel<<<grid_for(max_n * rv, kGatherThreads, device_sms() * 8), kGatherThreads, 0, stream>>>(
        words, n_dev, max_n, make_fastdiv((uint32_t)rv), reinterpret_cast<const int4*>(rows),
        reinterpret_cast<int4*>(out));
    return cuda_check(cudaGetLastError(), "moment_relay_scatter: launch");
}

moment_status launch_relay_push(moment_ctx_s* ctx, const int64_t* ids, const int64_t* qoff, const int64_t* qpos,
                                int64_t max_n, uint64_t* const* peer_inbox, int64_t* const* peer_count,
                                cudaStream_t stream) {
    if (!ctx->placement) return fail(MOMENT_EINVAL, "moment_relay_push: ctx has no placement map");
    if (ctx->world > MOMENT_MAX_WORLD) return fail(MOMENT_EUNSUPPORTED, "moment_relay_push: world > %d", MOMENT_MAX_WORLD);
    if (ctx->n_bins * (ctx->world - 1) > kMaxSegs) return fail(MOMENT_EUNSUPPORTED, "moment_relay_push: too many segments");
    PeerInboxes p{};
    for (int h = 0; h < ctx->world; h++) {
        if (h == ctx->rank) continue;
        if (!peer_inbox[h] || !peer_count[h] || (reinterpret_cast<uintptr_t>(peer_inbox[h]) & 15))
            return fail(MOMENT_EINVAL, "moment_relay_push: peer %d inbox / count null or inbox not 16-byte aligned", h);
        p.inbox[h] = peer_inbox[h];
        p.count[h] = peer_count[h];
    }
    const int grid = grid_for(std::max<int64_t>(max_n, 1), 256, device_sms() * 4);
    relay_push_kernel<<<grid, 256, 0, stream>>>(make_bins(ctx), ctx->placement, ids, qoff, qpos, ctx->n_bins, ctx->world,
                                                ctx->rank, p);
    return cuda_check(cudaGetLastError(), "moment_relay_push: launch");
}

moment_status launch_relay_serve_push(moment_ctx_s* ctx, const uint64_t* inbox, const int64_t* inbox_count, int64_t cap,
                                      void* const* peer_out, cudaStream_t stream) {
    if (ctx->world > MOMENT_MAX_WORLD) return fail(MOMENT_EUNSUPPORTED, "moment_relay_serve_push: world > %d", MOMENT_MAX_WORLD);
    PeerOuts o{};
    for (int g = 0; g < ctx->world; g++) {
        if (g == ctx->rank) continue;
        if (!peer_out[g] || (reinterpret_cast<uintptr_t>(peer_out[g]) & 15))
            return fail(MOMENT_EINVAL, "moment_relay_serve_push: peer %d output null or not 16-byte aligned", g);
        o.out[g] = reinterpret_cast<int4*>(peer_out[g]);
    }
    const int64_t rv = ctx->row_bytes / 16;
    // grid sized for the worst case (every source's full inbox); blocks without work exit at once
    const int grid = grid_for(std::max<int64_t>(cap * (ctx->world - 1) * rv, 1), kGatherThreads, device_sms() * 8);
    relay_serve_push_kernel<<<grid, kGatherThreads, 0, stream>>>(make_bins(ctx), inbox, inbox_count, cap, ctx->world,
                                                                 ctx->rank, make_fastdiv((uint32_t)rv),
                                                                 ctx->row_stride / 16, o);
    return cuda_check(cudaGetLastError(), "moment_relay_serve_push: launch");
}

// Kernel attributes, set once per device: every kernel of the library asks for the same shared-memory
// carveout (so consecutive kernels never force an L1/shared reconfiguration bubble on the SMs), and the
// bulk gather may use up to kBulkSmemMax bytes of dynamic shared memory.
moment_status configure_gather_kernels(int carveout) {
    const void* fns[] = {(const void*)gather_kernel, (const void*)gather_bulk_kernel<2>, (const void*)gather_bulk_kernel<4>,
                         (const void*)gather_bulk_kernel<6>, (const void*)gather_bulk_kernel<8>, (const void*)relay_kernel,
                         (const void*)bucket_count_kernel, (const void*)bucket_scan_kernel,
                         (const void*)bucket_route_kernel, (const void*)queue_count_kernel,
                         (const void*)queue_scan_kernel, (const void*)queue_scatter_kernel, (const void*)hotness_kernel};
    for (const void* f : fns)
        if (carveout >= 0)
            MOMENT_TRY(cuda_check(cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, carveout),
                                  "carveout attribute"));
    for (const void* f : {(const void*)gather_bulk_kernel<2>, (const void*)gather_bulk_kernel<4>,
                          (const void*)gather_bulk_kernel<6>, (const void*)gather_bulk_kernel<8>,
                          (const void*)gather_tma4_kernel<4, false>, (const void*)gather_tma4_kernel<4, true>,
                          (const void*)gather_tma4_kernel<4, false, 16>, (const void*)gather_tma4_kernel<4, true, 16>,
                          (const void*)gather_tma4_kernel<4, false, 8>, (const void*)gather_tma4_kernel<4, true, 8>})
        MOMENT_TRY(cuda_check(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmemMax),
                              "bulk gather smem attribute"));
    return MOMENT_OK;
}

moment_status launch_hotness(const int64_t* ids, const int64_t* n_dev, int64_t max_n, uint64_t* hot, cudaStream_t stream) {
    if (max_n <= 0) return MOMENT_OK;
    hotness_kernel<<<grid_for(max_n, 256, device_sms() * 8), 256, 0, stream>>>(ids, n_dev, max_n, hot);
    return cuda_check(cudaGetLastError(), "moment_hotness: launch");
}

}  // namespace moment
