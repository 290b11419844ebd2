// peer.cu — SURVEY.md §8(f) NEXT-4 / §8(e) "B200-native option": the cross-GPU reduction of a10
// fused into the compare path over NVLink peer memory instead of a separate ncclAllReduce.
//
// Every rank maps every peer's exchange block (CUDA IPC across processes, the raw pointer inside one
// process). Rank 0's block is the HOME of one run's first-mismatch indices, early-exit bounds and
// refutation counters: every rank's window kernels take home pointers, so a compare that finds a
// mismatch does its atomicMin (system scope) straight into rank 0's memory on the rare path, and a
// window refuted on any GPU publishes its bound where every GPU's skip test reads it (cross-GPU
// bounded early exit, Q9). The result is the same minimum the all-reduce computes (min over a
// partition of an ascending scan = first mismatch of the whole scan, SURVEY.md §8(c) "sharded oracle").
//
// One run on every rank:   reset (rank 0: home) -> barrier -> window kernels -> barrier
//                          -> gather (home first[] -> the plan's own first[]) -> barrier
// Barriers are one-warp kernels over per-source arrival slots: rank r stores its epoch into slot r of
// every peer (st.release.sys) and waits until every slot of its own block reaches the epoch
// (ld.acquire.sys), bounded by a %globaltimer timeout (60 s) that raises an error flag instead of
// hanging the GPU. The epoch lives in device memory and is advanced by the barrier kernel itself, so
// a run captured in a CUDA graph replays correctly.
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>
#include <stdlib.h>
#include <unistd.h>

#include "cec_internal.hpp"

namespace cec {
namespace {

inline const char *ck(cudaError_t e) { return e == cudaSuccess ? nullptr : cudaGetErrorString(e); }

__device__ __forceinline__ void st_release_sys(uint32_t *p, uint32_t v) {
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_sys(const unsigned long long *p) {
    uint64_t v;
    asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// own[0..PEER_MAX) = arrival slots (slot s = last epoch signalled by rank s), own[PEER_EPOCH] = this
// rank's epoch, own[PEER_ERR] = error flag (1 = a barrier timed out)
__global__ void peer_barrier(PeerPtrs pp, uint32_t *own, int rank, int world, uint64_t timeout_ns) {
    const int l = threadIdx.x;
    const uint32_t e = own[PEER_EPOCH] + 1u;  // written only by this kernel, stream-ordered
    if (l < world) {
        __threadfence_system();  // this rank's earlier writes before the signal
        st_release_sys(pp.slots[l] + rank, e);
        const uint64_t t0 = globaltimer();
        while ((int32_t)(ld_acquire_sys(own + l) - e) < 0) {
            if (globaltimer() - t0 > timeout_ns) {  // a peer never arrived (default 60 s)
                atomicExch(own + PEER_ERR, 1u);
                break;
            }
            __nanosleep(64);
        }
    }
    __syncwarp();
    if (l == 0) own[PEER_EPOCH] = e;
}

__global__ void peer_gather(const unsigned long long *home, unsigned long long *local, uint32_t n) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        local[i] = ld_relaxed_sys(home + i);
}

struct PeerBlob {  // CEC_PEER_BLOB_BYTES (128) on the wire
    uint32_t magic, pid;
    int32_t device, rank, world, pad;
    uint64_t ptr, bytes;
    cudaIpcMemHandle_t h;  // 64 B
    char bus[16];          // PCI bus id of the exporting device (process-independent device identity)
};
static_assert(sizeof(PeerBlob) <= 128, "peer blob");
constexpr uint32_t PEER_MAGIC = 0xCEC0BEEFu;

}  // namespace

size_t peer_block_bytes(uint32_t cap_cmp, uint32_t cap_win) {
    return PEER_HDR_BYTES + 8ull * cap_cmp + 8ull * cap_win + 4ull * cap_win;
}

const char *peer_export(PeerState &ps, int device, int rank, int world, void *blob128) {
    const char *e;
    if (!ps.own) {
        const size_t bytes = peer_block_bytes(ps.cap_cmp, ps.cap_win);
        if ((e = ck(cudaMalloc(&ps.own, bytes)))) return e;  // cudaMalloc: IPC-exportable
        if ((e = ck(cudaMemset(ps.own, 0, bytes)))) return e;
        if ((e = ck(cudaDeviceSynchronize()))) return e;
        ps.bytes = bytes;
    }
    PeerBlob b;
    memset(&b, 0, sizeof b);
    b.magic = PEER_MAGIC;
    b.pid = (uint32_t)getpid();
    b.device = device;
    b.rank = rank;
    b.world = world;
    b.ptr = (uint64_t)(uintptr_t)ps.own;
    b.bytes = ps.bytes;
    if ((e = ck(cudaIpcGetMemHandle(&b.h, ps.own)))) return e;
    if ((e = ck(cudaDeviceGetPCIBusId(b.bus, (int)sizeof b.bus, device)))) return e;
    memset(blob128, 0, 128);
    memcpy(blob128, &b, sizeof b);
    return nullptr;
}

const char *peer_import(PeerState &ps, int device, int rank, int world, const void *blobs) {
    if (!ps.own) return "cec_peer_export must be called before cec_peer_import";
    if (world < 2 || world > PEER_MAX) return "peer mode needs 2 <= world <= 8";
    const char *e;
    for (int r = 0; r < world; ++r) {
        PeerBlob b;
        memcpy(&b, (const char *)blobs + 128 * r, sizeof b);
        if (b.magic != PEER_MAGIC || b.rank != r || b.world != world || b.bytes != ps.bytes)
            return "peer blob mismatch (rank order, world or block size)";
        void *p = nullptr;
        if (r != rank) {
            // the home arrays take system-scope atomics from every rank: a peer on ANOTHER device
            // must be reachable with native P2P atomics (NVLink), else the import fails (the caller
            // then uses the NCCL all-reduce)
            char bus[17];
            memcpy(bus, b.bus, 16);
            bus[16] = 0;
            int pdev = -1;
            if (cudaDeviceGetByPCIBusId(&pdev, bus) != cudaSuccess) {
                cudaGetLastError();
                return "peer device not visible in this process (PCI bus id lookup failed)";
            }
            if (pdev != device) {
                int atom = 0, access = 0;
                if ((e = ck(cudaDeviceGetP2PAttribute(&access, cudaDevP2PAttrAccessSupported, device, pdev)))) return e;
                if ((e = ck(cudaDeviceGetP2PAttribute(&atom, cudaDevP2PAttrNativeAtomicSupported, device, pdev))))
                    return e;
                if (!access || !atom) return "no native P2P atomics between this device and a peer";
            }
        }
        if (r == rank) {
            p = ps.own;
        } else if (b.pid == (uint32_t)getpid()) {  // same process: the raw pointer (IPC refuses it)
            p = (void *)(uintptr_t)b.ptr;
            if (b.device != device) {
                const cudaError_t pe = cudaDeviceEnablePeerAccess(b.device, 0);
                if (pe != cudaSuccess && pe != cudaErrorPeerAccessAlreadyEnabled) return cudaGetErrorString(pe);
                cudaGetLastError();
            }
        } else {
            if ((e = ck(cudaIpcOpenMemHandle(&p, b.h, cudaIpcMemLazyEnablePeerAccess)))) return e;
            ps.opened[r] = p;
        }
        ps.peer[r] = p;
    }
    ps.rank = rank;
    ps.world = world;
    // a rank may still be planning / JIT-compiling while its peers wait at a barrier; only a peer
    // that is gone should trip the flag (CEC_PEER_TIMEOUT_S, default 60 s)
    ps.timeout_ns = 60000000000ull;
    if (const char *t = getenv("CEC_PEER_TIMEOUT_S")) ps.timeout_ns = (uint64_t)(atof(t) * 1e9);
    ps.on = true;
    ++ps.gen;
    return nullptr;
}

void peer_close(PeerState &ps) {
    for (int r = 0; r < PEER_MAX; ++r)
        if (ps.opened[r]) cudaIpcCloseMemHandle(ps.opened[r]);
    if (ps.own) cudaFree(ps.own);
    ps = PeerState{};
}

PeerRun peer_run_of(const PeerState &ps, unsigned long long *local_first) {
    PeerRun pr;
    pr.on = ps.on;
    pr.rank = ps.rank;
    pr.world = ps.world;
    for (int r = 0; r < ps.world; ++r) pr.slots.slots[r] = (uint32_t *)ps.peer[r];
    pr.own = (uint32_t *)ps.own;
    char *home = (char *)ps.peer[0];
    pr.home_first = (unsigned long long *)(home + PEER_HDR_BYTES);
    pr.home_bound = pr.home_first + ps.cap_cmp;
    pr.home_neq = (uint32_t *)(pr.home_bound + ps.cap_win);
    pr.local_first = local_first;
    pr.timeout_ns = ps.timeout_ns;
    pr.host_barrier = ps.host_barrier;
    pr.host_user = ps.host_user;
    return pr;
}

const char *peer_barrier_launch(const PeerRun &pr, void *stream) {
    if (pr.host_barrier) {
        // several ranks emulated on ONE device (cec_peer_host_barrier): kernels that wait on one
        // another must not be separate launches on one GPU (nothing makes them co-resident;
        // B200_PROFILING.md), so the barrier is this rank's work drained + the caller's host barrier
        const char *e = ck(cudaStreamSynchronize((cudaStream_t)stream));
        if (e) return e;
        pr.host_barrier(pr.host_user);
        return nullptr;
    }
    peer_barrier<<<1, 32, 0, (cudaStream_t)stream>>>(pr.slots, pr.own, pr.rank, pr.world, pr.timeout_ns);
    return ck(cudaGetLastError());
}

const char *peer_gather_launch(const PeerRun &pr, uint32_t n, void *stream) {
    if (!n) return nullptr;
    const uint32_t blocks = (n + 255) / 256 < 148 ? (n + 255) / 256 : 148;
    peer_gather<<<blocks, 256, 0, (cudaStream_t)stream>>>(pr.home_first, pr.local_first, n);
    return ck(cudaGetLastError());
}

const char *peer_error(const PeerState &ps, void *stream, bool *timed_out) {
    uint32_t f = 0;
    const char *e = ck(cudaMemcpyAsync(&f, (uint32_t *)ps.own + PEER_ERR, 4, cudaMemcpyDeviceToHost,
                                       (cudaStream_t)stream));
    if (!e) e = ck(cudaStreamSynchronize((cudaStream_t)stream));
    *timed_out = f != 0;
    return e;
}

}  // namespace cec
