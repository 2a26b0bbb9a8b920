// signal.cu — device-side barrier of the one-process-per-GPU exchange over peer memory (SURVEY 8(e):
// "symmetric-memory signal barrier per phase"; the relay path of P:L391-393). Each rank owns a flag word per
// peer (flags[world], CUDA-IPC mapped by the others). Arriving = a system-scope release store of the phase's
// epoch into every peer's slot for this rank; leaving = acquire loads until every peer's slot here holds the
// epoch. Enqueued on the stream, so the exchange needs no host synchronisation and can sit inside a CUDA graph.
#include <cuda_runtime.h>

#include <cstdint>

#include "ctx.h"
#include "moment.h"
#include "status.h"

using namespace moment;

namespace {

struct PeerFlags {
    uint64_t* p[MOMENT_MAX_WORLD];
};

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__global__ void signal_barrier_kernel(PeerFlags peer, int world, int rank, const uint64_t* flags, uint64_t epoch,
                                      int64_t timeout_ns, int32_t* status) {
    const int h = threadIdx.x;
    if (h < world && h != rank) {
        // every write this stream made before the barrier (earlier kernels' peer stores included) is ordered
        // before the flag: a system-scope fence, then the release store
        asm volatile("fence.sc.sys;" ::: "memory");
        st_release_sys(peer.p[h], epoch);
        const uint64_t t0 = globaltimer();
        unsigned ns = 32;
        while (ld_acquire_sys(flags + h) < epoch) {
            if ((int64_t)(globaltimer() - t0) > timeout_ns) {
                if (status) atomicExch(status, (int32_t)MOMENT_ETIMEDOUT);
                break;
            }
            __nanosleep(ns);
            ns = ns < 4096 ? ns * 2 : ns;
        }
    }
    __syncthreads();
}

// The same barrier with its epoch in device memory: every thread reads the counter, waits on epoch + 1, and
// thread 0 stores epoch + 1 back once all have left. Barriers on one stream run one after another, so each
// sees the previous one's value; a captured graph replays with fresh epochs.
__global__ void signal_barrier_dev_kernel(PeerFlags peer, int world, int rank, const uint64_t* flags,
                                          uint64_t* epoch_ctr, int64_t timeout_ns, int32_t* status) {
    const uint64_t epoch = *reinterpret_cast<volatile uint64_t*>(epoch_ctr) + 1;
    const int h = threadIdx.x;
    if (h < world && h != rank) {
        asm volatile("fence.sc.sys;" ::: "memory");
        st_release_sys(peer.p[h], epoch);
        const uint64_t t0 = globaltimer();
        unsigned ns = 32;
        while (ld_acquire_sys(flags + h) < epoch) {
            if ((int64_t)(globaltimer() - t0) > timeout_ns) {
                atomicExch(status, (int32_t)MOMENT_ETIMEDOUT);
                break;
            }
            __nanosleep(ns);
            ns = ns < 4096 ? ns * 2 : ns;
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) *epoch_ctr = epoch;
}

}  // namespace

namespace moment {

moment_status launch_signal_barrier_dev(const moment_ctx_s* c, cudaStream_t stream) {
    if (c->world == 1) return MOMENT_OK;
    PeerFlags pf{};
    for (int h = 0; h < c->world; h++) pf.p[h] = h == c->rank ? nullptr : c->ex.peer_flag[h];
    signal_barrier_dev_kernel<<<1, 64, 0, stream>>>(pf, c->world, c->rank, c->ex.flags, c->d_epoch, c->ex.timeout_ns,
                                                     c->d_xstatus);
    return cuda_check(cudaGetLastError(), "exchange barrier: launch");
}

}  // namespace moment

extern "C" moment_status moment_signal_barrier(int32_t world, int32_t rank, uint64_t* const* peer_flags,
                                               const uint64_t* flags, uint64_t epoch, int64_t timeout_ns,
                                               int32_t* status_dev, void* stream) {
    if (world < 1 || world > MOMENT_MAX_WORLD || rank < 0 || rank >= world)
        return fail(MOMENT_EINVAL, "moment_signal_barrier: rank %d / world %d out of range", rank, world);
    if (world > 1 && (!peer_flags || !flags)) return fail(MOMENT_EINVAL, "moment_signal_barrier: null argument");
    if (epoch == 0 || timeout_ns <= 0) return fail(MOMENT_EINVAL, "moment_signal_barrier: epoch and timeout must be > 0");
    PeerFlags pf{};
    for (int h = 0; h < world; h++) {
        if (h == rank) continue;
        if (!peer_flags[h]) return fail(MOMENT_EINVAL, "moment_signal_barrier: peer_flags[%d] is null", h);
        pf.p[h] = peer_flags[h];
    }
    MOMENT_TRY(cuda_pending("moment_signal_barrier: pending CUDA error"));
    if (world == 1) return MOMENT_OK;
    signal_barrier_kernel<<<1, 64, 0, static_cast<cudaStream_t>(stream)>>>(pf, world, rank, flags, epoch, timeout_ns,
                                                                            status_dev);
    return cuda_check(cudaGetLastError(), "moment_signal_barrier: launch");
}
