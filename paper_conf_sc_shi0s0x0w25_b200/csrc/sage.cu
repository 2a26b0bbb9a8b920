// sage.cu — the consumer of a sampled batch: GraphSAGE mean aggregation over one
// sampled block, forward and backward (Eq. 1: h_v^l depends on the aggregate of h_u^{l-1} over
// the sampled neighbours; the paper trains GraphSAGE with hidden 256). The dense parts of the layer
// (the two weight GEMMs, ReLU, loss) are plain library GEMMs in the caller; these kernels are the sparse,
// HBM-bound part: random source rows read once per edge (forward) or scattered once per edge (backward).
//
// Layout: x[n_src][ld_x] (fp32 or bf16), a block = the per-hop offsets int64[n_dst + 1] (relative to the
// block's first edge) and src int32[E] of moment_sample; out[n_dst][ld_out] of the same dtype as x.
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "ctx.h"
#include "moment.h"
#include "status.h"

using namespace moment;

namespace {

constexpr int kWarps = 8;  // warps per block; one dst row per warp

__device__ __forceinline__ void acc_vec(float* a, const uint4& v, int32_t dtype) {
    if (dtype == MOMENT_DTYPE_F32) {
        a[0] += __uint_as_float(v.x);
        a[1] += __uint_as_float(v.y);
        a[2] += __uint_as_float(v.z);
        a[3] += __uint_as_float(v.w);
    } else {
        const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
        for (int q = 0; q < 4; q++) {
            a[2 * q] += __uint_as_float(w[q] << 16);
            a[2 * q + 1] += __uint_as_float(w[q] & 0xFFFF0000u);
        }
    }
}

__device__ __forceinline__ uint4 pack_vec(const float* a, float scale, int32_t dtype) {
    uint4 r;
    if (dtype == MOMENT_DTYPE_F32) {
        r.x = __float_as_uint(a[0] * scale);
        r.y = __float_as_uint(a[1] * scale);
        r.z = __float_as_uint(a[2] * scale);
        r.w = __float_as_uint(a[3] * scale);
    } else {
        uint32_t w[4];
#pragma unroll
        for (int q = 0; q < 4; q++) {
            const __nv_bfloat162 h = __floats2bfloat162_rn(a[2 * q] * scale, a[2 * q + 1] * scale);
            w[q] = *reinterpret_cast<const uint32_t*>(&h);
        }
        r = make_uint4(w[0], w[1], w[2], w[3]);
    }
    return r;
}

// out[i] = mean over the block's edges of x[src[e]]. One warp per dst row; lane l owns the 16-byte vectors
// l, l + 32, ... (VPL of them) of the row; four edges' rows in flight per lane (independent LDG.128).
template <int VPL>
__global__ void __launch_bounds__(32 * kWarps) sage_mean_kernel(const char* __restrict__ x, int64_t ldx_b,
                                                                 int32_t dtype, int32_t nv,
                                                                 const int64_t* __restrict__ offsets,
                                                                 const int32_t* __restrict__ src, int64_t n_dst,
                                                                 char* __restrict__ out, int64_t ldo_b) {
    const int lane = threadIdx.x & 31;
    const int64_t warp0 = (int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5);
    const int64_t nwarps = (int64_t)gridDim.x * kWarps;
    for (int64_t i = warp0; i < n_dst; i += nwarps) {
        const int64_t e0 = offsets[i], e1 = offsets[i + 1];
        float a[VPL][8];
#pragma unroll
        for (int v = 0; v < VPL; v++)
#pragma unroll
            for (int q = 0; q < 8; q++) a[v][q] = 0.f;
        for (int64_t eb = e0; eb < e1; eb += 32) {
            const int cnt = (int)min((int64_t)32, e1 - eb);
            const int32_t my = lane < cnt ? __ldg(src + eb + lane) : 0;
            int j = 0;
            for (; j + 4 <= cnt; j += 4) {
                uint4 r[4][VPL];
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    const int32_t s = __shfl_sync(0xffffffffu, my, j + u);
                    const uint4* row = reinterpret_cast<const uint4*>(x + (int64_t)s * ldx_b);
#pragma unroll
                    for (int v = 0; v < VPL; v++) {
                        const int c = lane + 32 * v;
                        r[u][v] = c < nv ? __ldg(row + c) : make_uint4(0, 0, 0, 0);
                    }
                }
#pragma unroll
                for (int u = 0; u < 4; u++)
#pragma unroll
                    for (int v = 0; v < VPL; v++) acc_vec(a[v], r[u][v], dtype);
            }
            for (; j < cnt; j++) {
                const int32_t s = __shfl_sync(0xffffffffu, my, j);
                const uint4* row = reinterpret_cast<const uint4*>(x + (int64_t)s * ldx_b);
#pragma unroll
                for (int v = 0; v < VPL; v++) {
                    const int c = lane + 32 * v;
                    if (c < nv) acc_vec(a[v], __ldg(row + c), dtype);
                }
            }
        }
        const float scale = e1 > e0 ? 1.f / (float)(e1 - e0) : 0.f;
        uint4* orow = reinterpret_cast<uint4*>(out + i * ldo_b);
#pragma unroll
        for (int v = 0; v < VPL; v++) {
            const int c = lane + 32 * v;
            if (c < nv) orow[c] = pack_vec(a[v], scale, dtype);
        }
    }
}

// grad_x[src[e]] += grad_out[i] / deg_i for every edge e of row i: fp32 vector atomics (RED.ADD.F32x4).
template <int VPL>
__global__ void __launch_bounds__(32 * kWarps) sage_mean_bwd_kernel(const char* __restrict__ g, int64_t ldg_b,
                                                                     int32_t dtype, int32_t nv,
                                                                     const int64_t* __restrict__ offsets,
                                                                     const int32_t* __restrict__ src,
                                                                     int64_t n_dst, float* __restrict__ gx,
                                                                     int64_t ldgx) {
    const int lane = threadIdx.x & 31;
    const int64_t warp0 = (int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5);
    const int64_t nwarps = (int64_t)gridDim.x * kWarps;
    const int fpv = dtype == MOMENT_DTYPE_F32 ? 4 : 8;  // floats per 16-byte input vector
    for (int64_t i = warp0; i < n_dst; i += nwarps) {
        const int64_t e0 = offsets[i], e1 = offsets[i + 1];
        if (e1 == e0) continue;
        const float scale = 1.f / (float)(e1 - e0);
        float a[VPL][8];
        const uint4* grow = reinterpret_cast<const uint4*>(g + i * ldg_b);
#pragma unroll
        for (int v = 0; v < VPL; v++) {
#pragma unroll
            for (int q = 0; q < 8; q++) a[v][q] = 0.f;
            const int c = lane + 32 * v;
            if (c < nv) acc_vec(a[v], __ldg(grow + c), dtype);
#pragma unroll
            for (int q = 0; q < 8; q++) a[v][q] *= scale;
        }
        for (int64_t eb = e0; eb < e1; eb += 32) {
            const int cnt = (int)min((int64_t)32, e1 - eb);
            const int32_t my = lane < cnt ? __ldg(src + eb + lane) : 0;
            for (int j = 0; j < cnt; j++) {
                const int32_t s = __shfl_sync(0xffffffffu, my, j);
                float* row = gx + (int64_t)s * ldgx;
#pragma unroll
                for (int v = 0; v < VPL; v++) {
                    const int c = lane + 32 * v;
                    if (c >= nv) continue;
                    float4* p = reinterpret_cast<float4*>(row + (int64_t)c * fpv);
                    atomicAdd(p, make_float4(a[v][0], a[v][1], a[v][2], a[v][3]));
                    if (fpv == 8) atomicAdd(p + 1, make_float4(a[v][4], a[v][5], a[v][6], a[v][7]));
                }
            }
        }
    }
}

moment_status check_args(const void* x, int64_t ld_x, int32_t dtype, int64_t dim, const int64_t* offsets,
                         const int32_t* src, int64_t n_dst, const void* out, int64_t ld_out, int32_t* nv,
                         const char* who) {
    if (n_dst < 0 || dim <= 0) return fail(MOMENT_EINVAL, "%s: n_dst %lld / dim %lld out of range", who, (long long)n_dst, (long long)dim);
    if (dtype != MOMENT_DTYPE_F32 && dtype != MOMENT_DTYPE_BF16) return fail(MOMENT_EINVAL, "%s: dtype %d", who, dtype);
    const int64_t es = dtype == MOMENT_DTYPE_F32 ? 4 : 2;
    if ((dim * es) % 16 != 0) return fail(MOMENT_EINVAL, "%s: a row (%lld bytes) must be a multiple of 16 bytes", who, (long long)(dim * es));
    if (dim * es > 32 * 16 * 4) return fail(MOMENT_EUNSUPPORTED, "%s: rows above 2048 bytes", who);
    if (ld_x < dim || ld_out < dim || (ld_x * es) % 16 || (ld_out * es) % 16)
        return fail(MOMENT_EINVAL, "%s: leading dimensions must be >= dim and 16-byte multiples", who);
    if (n_dst > 0 && (!x || !offsets || !src || !out)) return fail(MOMENT_EINVAL, "%s: null argument", who);
    if (((uintptr_t)x | (uintptr_t)out) & 15) return fail(MOMENT_EINVAL, "%s: x and out must be 16-byte aligned", who);
    *nv = (int32_t)(dim * es / 16);
    return MOMENT_OK;
}

int grid_for(int64_t n_dst) {
    return (int)std::max<int64_t>(1, std::min<int64_t>((n_dst + kWarps - 1) / kWarps, device_sms() * 8));
}

}  // namespace

extern "C" moment_status moment_sage_mean(const void* x, int64_t ld_x, int32_t dtype, int64_t dim,
                                          const int64_t* offsets, const int32_t* src, int64_t n_dst, void* out,
                                          int64_t ld_out, void* stream) {
    int32_t nv = 0;
    MOMENT_TRY(check_args(x, ld_x, dtype, dim, offsets, src, n_dst, out, ld_out, &nv, "moment_sage_mean"));
    MOMENT_TRY(cuda_pending("moment_sage_mean: pending CUDA error"));
    if (n_dst == 0) return MOMENT_OK;
    const int64_t es = dtype == MOMENT_DTYPE_F32 ? 4 : 2;
    auto st = static_cast<cudaStream_t>(stream);
    const int grid = grid_for(n_dst);
    const int vpl = (nv + 31) / 32;
    const char* xb = static_cast<const char*>(x);
    char* ob = static_cast<char*>(out);
    if (vpl == 1) sage_mean_kernel<1><<<grid, 32 * kWarps, 0, st>>>(xb, ld_x * es, dtype, nv, offsets, src, n_dst, ob, ld_out * es);
    else if (vpl == 2) sage_mean_kernel<2><<<grid, 32 * kWarps, 0, st>>>(xb, ld_x * es, dtype, nv, offsets, src, n_dst, ob, ld_out * es);
    else sage_mean_kernel<4><<<grid, 32 * kWarps, 0, st>>>(xb, ld_x * es, dtype, nv, offsets, src, n_dst, ob, ld_out * es);
    return cuda_check(cudaGetLastError(), "moment_sage_mean: launch");
}

extern "C" moment_status moment_sage_mean_backward(const void* grad_out, int64_t ld_g, int32_t dtype, int64_t dim,
                                                   const int64_t* offsets, const int32_t* src, int64_t n_dst,
                                                   float* grad_x, int64_t ld_gx, void* stream) {
    int32_t nv = 0;
    MOMENT_TRY(check_args(grad_out, ld_g, dtype, dim, offsets, src, n_dst, grad_x, ld_g, &nv,
                          "moment_sage_mean_backward"));
    if (ld_gx < dim || ld_gx % 4) return fail(MOMENT_EINVAL, "moment_sage_mean_backward: ld_gx must be >= dim, a multiple of 4");
    MOMENT_TRY(cuda_pending("moment_sage_mean_backward: pending CUDA error"));
    if (n_dst == 0) return MOMENT_OK;
    const int64_t es = dtype == MOMENT_DTYPE_F32 ? 4 : 2;
    auto st = static_cast<cudaStream_t>(stream);
    const int grid = grid_for(n_dst);
    const int vpl = (nv + 31) / 32;
    const char* gb = static_cast<const char*>(grad_out);
    if (vpl == 1) sage_mean_bwd_kernel<1><<<grid, 32 * kWarps, 0, st>>>(gb, ld_g * es, dtype, nv, offsets, src, n_dst, grad_x, ld_gx);
    else if (vpl == 2) sage_mean_bwd_kernel<2><<<grid, 32 * kWarps, 0, st>>>(gb, ld_g * es, dtype, nv, offsets, src, n_dst, grad_x, ld_gx);
    else sage_mean_bwd_kernel<4><<<grid, 32 * kWarps, 0, st>>>(gb, ld_g * es, dtype, nv, offsets, src, n_dst, grad_x, ld_gx);
    return cuda_check(cudaGetLastError(), "moment_sage_mean_backward: launch");
}
