// device_util.cuh — device-side building blocks: Philox4x32-10, block scan, decoupled look-back.
#pragma once
#include <cuda/atomic>
#include <cuda_runtime.h>

#include <cstdint>

namespace moment {
namespace dev {

// Philox4x32-10 (Salmon et al., SC '11): the counter-based stream the sampler draws from (R1).
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 k) {
#pragma unroll
    for (int r = 0; r < 10; r++) {
        const uint32_t lo0 = 0xD2511F53u * c.x, hi0 = __umulhi(0xD2511F53u, c.x);
        const uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = __umulhi(0xCD9E8D57u, c.z);
        c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
        k.x += 0x9E3779B9u;
        k.y += 0xBB67AE85u;
    }
    return c;
}

// draw(seed, v, h, i): word i & 3 of Philox(ctr = (lo v, hi v, h, i >> 2), key = (lo seed, hi seed)).
__device__ __forceinline__ uint32_t draw(uint64_t seed, int64_t v, int32_t h, int32_t i) {
    const uint4 r = philox4x32_10(make_uint4((uint32_t)v, (uint32_t)((uint64_t)v >> 32), (uint32_t)h, (uint32_t)(i >> 2)),
                                  make_uint2((uint32_t)seed, (uint32_t)(seed >> 32)));
    const int w = i & 3;
    return w == 0 ? r.x : (w == 1 ? r.y : (w == 2 ? r.z : r.w));
}

// Integer in [0, m) from a 32-bit draw: floor(r m / 2^32) (R2).
__device__ __forceinline__ uint32_t uniform(uint32_t r, uint32_t m) {
    return (uint32_t)(((uint64_t)r * (uint64_t)m) >> 32);
}

// Read-only random loads with a 64-byte L2 fetch size hint (the default fetches the whole 128-byte line a
// lone 4- or 8-byte read touches).
__device__ __forceinline__ int32_t ld_rand(const int32_t* p) {
    int32_t v;
    asm("ld.global.nc.L2::64B.b32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ int64_t ld_rand(const int64_t* p) {
    int64_t v;
    asm("ld.global.nc.L2::64B.b64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ uint64_t ld_rand(const uint64_t* p) {
    uint64_t v;
    asm("ld.global.nc.L2::64B.b64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}

// Block-wide exclusive scan of one int64 per thread (blockDim.x == NT, multiple of 32).
template <int NT>
__device__ __forceinline__ int64_t block_exclusive_scan(int64_t x, int64_t* total, int64_t* warp_sums) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int64_t incl = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        int64_t y = __shfl_up_sync(0xffffffffu, incl, d);
        if (lane >= d) incl += y;
    }
    if (lane == 31) warp_sums[wid] = incl;
    __syncthreads();
    if (wid == 0) {
        int64_t w = lane < NT / 32 ? warp_sums[lane] : 0;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            int64_t y = __shfl_up_sync(0xffffffffu, w, d);
            if (lane >= d) w += y;
        }
        if (lane < NT / 32) warp_sums[lane] = w;  // inclusive
    }
    __syncthreads();
    const int64_t warp_base = wid > 0 ? warp_sums[wid - 1] : 0;
    *total = warp_sums[NT / 32 - 1];
    return warp_base + incl - x;
}

// Decoupled look-back (single-pass chained scan). Descriptor: bits 62..63 = state (0 empty,
// 1 aggregate, 2 inclusive prefix), bits 0..61 = value. Called by one warp / block per tile; tiles are taken
// in increasing order through an atomic ticket, so every predecessor tile is owned by a running block.
constexpr uint64_t kFlagAgg = 1ull << 62, kFlagPrefix = 2ull << 62, kValMask = (1ull << 62) - 1;

// A descriptor carries its flag and its value in ONE 64-bit word written by one store, so readers need
// only coherence on that word: relaxed device-scope atomics (no fence, no L1 invalidate per poll).
__device__ __forceinline__ uint64_t ld_flag(const uint64_t* p) {
    return cuda::atomic_ref<unsigned long long, cuda::thread_scope_device>(
               *reinterpret_cast<unsigned long long*>(const_cast<uint64_t*>(p)))
        .load(cuda::memory_order_relaxed);
}
__device__ __forceinline__ void st_flag(uint64_t* p, uint64_t v) {
    cuda::atomic_ref<unsigned long long, cuda::thread_scope_device>(*reinterpret_cast<unsigned long long*>(p))
        .store(v, cuda::memory_order_relaxed);
}

// Warp-parallel decoupled look-back: called by ALL 32 lanes of one warp; inspects 32 predecessors per
// step (lane 0 = nearest), stops at the nearest inclusive prefix. Returns the exclusive prefix (all lanes).
__device__ __forceinline__ int64_t lookback_warp(uint64_t* status, int64_t tile, int64_t aggregate) {
    const int lane = threadIdx.x & 31;
    if (tile == 0) {
        if (lane == 0) st_flag(&status[0], kFlagPrefix | (uint64_t)aggregate);
        return 0;
    }
    if (lane == 0) st_flag(&status[tile], kFlagAgg | (uint64_t)aggregate);
    int64_t exclusive = 0;
    for (int64_t end = tile - 1;; end -= 32) {
        const int64_t j = end - lane;
        uint64_t s = kFlagPrefix;  // "before tile 0" acts as a zero prefix (never reached: tile 0 is a prefix)
        if (j >= 0) {
            s = ld_flag(&status[j]);
            while ((s & ~kValMask) == 0) {
                __nanosleep(64);
                s = ld_flag(&status[j]);
            }
        }
        const unsigned pre = __ballot_sync(0xffffffffu, (s & ~kValMask) == kFlagPrefix);
        const int stop = pre ? __ffs(pre) - 1 : 32;
        int64_t v = (lane <= stop && j >= 0) ? (int64_t)(s & kValMask) : 0;
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
        exclusive += v;
        if (pre) break;
    }
    if (lane == 0) st_flag(&status[tile], kFlagPrefix | (uint64_t)(exclusive + aggregate));
    return exclusive;
}

// Block-wide decoupled look-back: ALL NT threads call it; each step inspects NT predecessors at once
// (thread 0 = nearest), waits until each has published, and stops at the nearest inclusive prefix.
// Returns the exclusive prefix to every thread. `red` is NT/32 int64 of shared scratch, `flag` one int.
template <int NT>
__device__ __forceinline__ int64_t lookback_block(uint64_t* status, int64_t tile, int64_t aggregate, int64_t* red,
                                                  int* nearest) {
    if (tile == 0) {
        if (threadIdx.x == 0) st_flag(&status[0], kFlagPrefix | (uint64_t)aggregate);
        return 0;
    }
    if (threadIdx.x == 0) st_flag(&status[tile], kFlagAgg | (uint64_t)aggregate);
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int64_t exclusive = 0;
    for (int64_t end = tile - 1;; end -= NT) {
        const int64_t j = end - threadIdx.x;
        uint64_t s = 0;
        if (j >= 0) {
            s = ld_flag(&status[j]);
            while ((s & ~kValMask) == 0) {  // back off: polling warps must not crowd out working ones
                __nanosleep(64);
                s = ld_flag(&status[j]);
            }
        }
        if (threadIdx.x == 0) *nearest = NT;
        __syncthreads();
        if (j >= 0 && (s & ~kValMask) == kFlagPrefix) atomicMin(nearest, (int)threadIdx.x);
        __syncthreads();
        const int stop = *nearest;
        int64_t v = (j >= 0 && (int)threadIdx.x <= stop) ? (int64_t)(s & kValMask) : 0;
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
        if (lane == 0) red[wid] = v;
        __syncthreads();
        int64_t sum = 0;
#pragma unroll
        for (int w = 0; w < NT / 32; w++) sum += red[w];
        exclusive += sum;
        __syncthreads();
        if (stop < NT || end - NT < 0) break;
    }
    if (threadIdx.x == 0) st_flag(&status[tile], kFlagPrefix | (uint64_t)(exclusive + aggregate));
    return exclusive;
}

}  // namespace dev
}  // namespace moment
