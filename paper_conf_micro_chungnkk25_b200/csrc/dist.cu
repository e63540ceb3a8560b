// dist.cu -- multi-GPU plan: one process (or thread) per GPU,
// trace rows sharded by row range.  The path shards naturally by kernel id:
// ROOT decisions depend only on a cluster's own rows, so after
// one all-to-all that gives every rank whole kernel groups, everything is
// local except the two global KKT scalars (T and Ssum, reduced EXACTLY as
// integers) and the final estimate sums.  Kernel ranges are contiguous and
// rows arrive in global row order, so leaves, ordinals, Philox counters and
// sample rows are identical for every GPU count.
//
// Collectives go through class Comm: NCCL (dlopen'ed libnccl.so.2, device
// buffers over NVLink/NVSwitch) or a loopback group of threads sharing one
// GPU (single-GPU tests of the multi-rank logic).
#include <dlfcn.h>

#include <chrono>
#include <condition_variable>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <memory>
#include <mutex>
#include <vector>

#include "internal.h"
#include "nccl.h"

namespace sr {

// ---------------------------------------------------------------- communicators
// Seconds a rank waits for its peers (a collective, a barrier) before giving up
// with STEM_E_NCCL: STEMROOT_COMM_TIMEOUT_S, default 600.
static double comm_timeout_s() {
    static double v = -1.0;
    if (v < 0.0) {
        const char *e = getenv("STEMROOT_COMM_TIMEOUT_S");
        v = e ? atof(e) : 600.0;
        if (!(v > 0.0)) v = 600.0;
    }
    return v;
}

class Comm {
  public:
    int rank = 0, world = 1, device = 0;
    bool broken = false;   // a peer failed or timed out: every later call returns STEM_E_NCCL
    virtual ~Comm() {}
    // wait for everything queued on st, collectives included; STEM_E_NCCL on a
    // communicator error or after comm_timeout_s() (the communicator is then unusable)
    virtual int wait(cudaStream_t st) {
        if (broken) return STEM_E_NCCL;
        CK(cudaStreamSynchronize(st));
        return STEM_OK;
    }
    // in-place sum over ranks of a device buffer (u64 or f64)
    virtual int allreduce(void *buf, size_t count, bool f64, cudaStream_t st) = 0;
    // host arrays: all[r * count + i] = rank r's mine[i]
    virtual int allgather_host(const uint64_t *mine, size_t count, uint64_t *all, cudaStream_t st) = 0;
    // device buffers; counts/displacements are host arrays of `world` elements (units of elem bytes)
    // Collective: every rank passes nptr device buffers of its own; peers[r *
    // nptr + i] receives rank r's buffer i as a pointer this rank's kernels can
    // store to (peer memory over NVLink; its own buffers for r == rank).
    // STEM_E_CUDA (on every rank) when peer access is not possible.
    virtual int window(void *const *mine, int nptr, void **peers, cudaStream_t st) = 0;
    virtual int alltoallv(const void *send, const uint64_t *scnt, const uint64_t *sdsp, void *recv,
                          const uint64_t *rcnt, const uint64_t *rdsp, size_t elem, cudaStream_t st) = 0;
};

struct NcclApi {
    bool ok = false;
    ncclResult_t (*getUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*commInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*allReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*allGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*groupStart)() = nullptr;
    ncclResult_t (*groupEnd)() = nullptr;
    ncclResult_t (*getAsyncError)(ncclComm_t, ncclResult_t *) = nullptr;   // optional
    ncclResult_t (*commAbort)(ncclComm_t) = nullptr;                         // optional
};

static NcclApi &nccl() {
    static NcclApi api = [] {
        NcclApi a;
        void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) return a;
        a.getUniqueId = (decltype(a.getUniqueId))dlsym(h, "ncclGetUniqueId");
        a.commInitRank = (decltype(a.commInitRank))dlsym(h, "ncclCommInitRank");
        a.commDestroy = (decltype(a.commDestroy))dlsym(h, "ncclCommDestroy");
        a.allReduce = (decltype(a.allReduce))dlsym(h, "ncclAllReduce");
        a.allGather = (decltype(a.allGather))dlsym(h, "ncclAllGather");
        a.send = (decltype(a.send))dlsym(h, "ncclSend");
        a.recv = (decltype(a.recv))dlsym(h, "ncclRecv");
        a.groupStart = (decltype(a.groupStart))dlsym(h, "ncclGroupStart");
        a.groupEnd = (decltype(a.groupEnd))dlsym(h, "ncclGroupEnd");
        a.getAsyncError = (decltype(a.getAsyncError))dlsym(h, "ncclCommGetAsyncError");
        a.commAbort = (decltype(a.commAbort))dlsym(h, "ncclCommAbort");
        a.ok = a.getUniqueId && a.commInitRank && a.commDestroy && a.allReduce && a.allGather && a.send &&
               a.recv && a.groupStart && a.groupEnd;
        return a;
    }();
    return api;
}

#define NK(x)                                                  \
    do {                                                       \
        if (broken) return STEM_E_NCCL;                        \
        if ((x) != ncclSuccess) { fail(); return STEM_E_NCCL; } \
    } while (0)

class NcclComm : public Comm {
  public:
    ncclComm_t comm = nullptr;
    uint64_t *stage = nullptr;
    size_t stage_cap = 0;
    struct IpcMap {
        cudaIpcMemHandle_t h;
        void *p = nullptr;
    };
    std::vector<IpcMap> ipc;   // [world * nptr] peer buffers opened by CUDA IPC (cached by handle)
    ~NcclComm() override {
        for (auto &m : ipc)
            if (m.p) cudaIpcCloseMemHandle(m.p);
        if (comm) nccl().commDestroy(comm);
        if (stage) cudaFree(stage);
    }
    // CUDA IPC: handles allgathered, peers' buffers opened once per allocation
    int window(void *const *mine, int nptr, void **peers, cudaStream_t st) override {
        if (broken) return STEM_E_NCCL;
        constexpr int HW = (int)(sizeof(cudaIpcMemHandle_t) / 8);   // 64-byte handle = 8 words
        std::vector<uint64_t> my((size_t)nptr * HW + 1, 0), all((size_t)world * (nptr * HW + 1));
        int st_local = STEM_OK;
        for (int i = 0; i < nptr && st_local == STEM_OK; i++) {
            cudaIpcMemHandle_t h;
            if (cudaIpcGetMemHandle(&h, mine[i]) != cudaSuccess) { cudaGetLastError(); st_local = STEM_E_CUDA; }
            else memcpy(&my[(size_t)i * HW], &h, sizeof(h));
        }
        my[(size_t)nptr * HW] = (uint64_t)(int64_t)st_local;
        CKS(allgather_host(my.data(), my.size(), all.data(), st));
        for (int r = 0; r < world; r++)
            if ((int64_t)all[(size_t)r * my.size() + nptr * HW] != STEM_OK) return STEM_E_CUDA;
        if (ipc.size() != (size_t)world * nptr) {
            for (auto &m : ipc)
                if (m.p) cudaIpcCloseMemHandle(m.p);
            ipc.assign((size_t)world * nptr, IpcMap{});
        }
        for (int r = 0; r < world && st_local == STEM_OK; r++)
            for (int i = 0; i < nptr; i++) {
                if (r == rank) { peers[(size_t)r * nptr + i] = mine[i]; continue; }
                IpcMap &m = ipc[(size_t)r * nptr + i];
                const void *hr = &all[(size_t)r * my.size() + (size_t)i * HW];
                if (!m.p || memcmp(&m.h, hr, sizeof(m.h)) != 0) {
                    if (m.p) cudaIpcCloseMemHandle(m.p);
                    m.p = nullptr;
                    memcpy(&m.h, hr, sizeof(m.h));
                    if (cudaIpcOpenMemHandle(&m.p, m.h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
                        cudaGetLastError();
                        m.p = nullptr;
                        st_local = STEM_E_CUDA;
                        break;
                    }
                }
                peers[(size_t)r * nptr + i] = m.p;
            }
        // every rank learns whether every rank could open every peer
        uint64_t flag = (uint64_t)(int64_t)st_local;
        std::vector<uint64_t> flags(world);
        CKS(allgather_host(&flag, 1, flags.data(), st));
        for (int r = 0; r < world; r++)
            if ((int64_t)flags[r] != STEM_OK) return STEM_E_CUDA;
        return STEM_OK;
    }
    void fail() {   // abort the communicator: queued NCCL kernels terminate, later calls fail fast
        if (comm && nccl().commAbort) nccl().commAbort(comm);
        else if (comm) nccl().commDestroy(comm);
        comm = nullptr;
        broken = true;
    }
    // Poll the stream and the communicator's asynchronous error state instead
    // of blocking in cudaStreamSynchronize: a lost or failed peer turns into
    // STEM_E_NCCL within comm_timeout_s() instead of a hang.
    int wait(cudaStream_t st) override {
        if (broken) return STEM_E_NCCL;
        const auto t0 = std::chrono::steady_clock::now();
        for (uint64_t it = 0;; it++) {
            const cudaError_t e = cudaStreamQuery(st);
            if (e == cudaSuccess) return STEM_OK;
            if (e != cudaErrorNotReady) {
                last_cuda_error() = e;
                return STEM_E_CUDA;
            }
            ncclResult_t ae = ncclSuccess;
            if (nccl().getAsyncError && nccl().getAsyncError(comm, &ae) == ncclSuccess && ae != ncclSuccess &&
                ae != ncclInProgress) {
                fail();
                return STEM_E_NCCL;
            }
            const double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
            if (el > comm_timeout_s()) {
                fail();
                return STEM_E_NCCL;
            }
            if (el > 2e-3) std::this_thread::sleep_for(std::chrono::microseconds(50));
        }
    }
    int allreduce(void *buf, size_t count, bool f64, cudaStream_t st) override {
        NK(nccl().allReduce(buf, buf, count, f64 ? ncclFloat64 : ncclUint64, ncclSum, comm, st));
        return STEM_OK;
    }
    int allgather_host(const uint64_t *mine, size_t count, uint64_t *all, cudaStream_t st) override {
        const size_t need = count * (world + 1) * sizeof(uint64_t);
        if (need > stage_cap) {
            if (stage) cudaFree(stage);
            stage = nullptr;
            CK(cudaMalloc((void **)&stage, need));
            stage_cap = need;
        }
        uint64_t *send = stage + count * world;
        CK(cudaMemcpyAsync(send, mine, count * sizeof(uint64_t), cudaMemcpyHostToDevice, st));
        NK(nccl().allGather(send, stage, count, ncclUint64, comm, st));
        CK(cudaMemcpyAsync(all, stage, count * world * sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        return wait(st);
    }
    int alltoallv(const void *send, const uint64_t *scnt, const uint64_t *sdsp, void *recv, const uint64_t *rcnt,
                  const uint64_t *rdsp, size_t elem, cudaStream_t st) override {
        NK(nccl().groupStart());
        for (int p = 0; p < world; p++) {
            if (scnt[p])
                NK(nccl().send((const char *)send + sdsp[p] * elem, scnt[p] * elem, ncclUint8, p, comm, st));
            if (rcnt[p]) NK(nccl().recv((char *)recv + rdsp[p] * elem, rcnt[p] * elem, ncclUint8, p, comm, st));
        }
        NK(nccl().groupEnd());
        return STEM_OK;
    }
};

// Loopback: `world` threads on one GPU, rendezvous on a host barrier, data moved
// by device-to-device copies / a summing kernel.
struct LoopGroup {
    int world;
    std::mutex m;
    std::condition_variable cv;
    int arrived = 0;
    uint64_t gen = 0;
    std::vector<const void *> ptr;
    std::vector<const uint64_t *> h0, h1;
    std::vector<void *const *> wptr;
    bool broken = false;
    explicit LoopGroup(int w) : world(w), ptr(w), h0(w), h1(w), wptr(w) {}
    // false when a member did not arrive within comm_timeout_s() (the group is then broken)
    bool barrier() {
        std::unique_lock<std::mutex> l(m);
        if (broken) return false;
        const uint64_t g = gen;
        if (++arrived == world) {
            arrived = 0;
            gen++;
            cv.notify_all();
            return true;
        }
        const auto dl = std::chrono::steady_clock::now() +
                        std::chrono::duration_cast<std::chrono::steady_clock::duration>(
                            std::chrono::duration<double>(comm_timeout_s()));
        if (!cv.wait_until(l, dl, [&] { return gen != g || broken; }) || broken) {
            broken = true;
            cv.notify_all();
            return false;
        }
        return true;
    }
};

constexpr int kMaxWorld = 64;
struct PtrSet { const void *p[kMaxWorld]; };

__global__ void sum_buffers_kernel(PtrSet ps, int world, size_t count, bool f64, void *out) {
    const size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= count) return;
    if (f64) {
        double s = 0.0;
        for (int r = 0; r < world; r++) s = __dadd_rn(s, ((const double *)ps.p[r])[i]);   // fixed rank order
        ((double *)out)[i] = s;
    } else {
        uint64_t s = 0;
        for (int r = 0; r < world; r++) s += ((const uint64_t *)ps.p[r])[i];
        ((uint64_t *)out)[i] = s;
    }
}

class LoopComm : public Comm {
  public:
    std::shared_ptr<LoopGroup> g;
    void *tmp = nullptr;
    size_t tmp_cap = 0;
    ~LoopComm() override {
        if (tmp) cudaFree(tmp);
    }
    int allreduce(void *buf, size_t count, bool f64, cudaStream_t st) override {
        if (count * 8 > tmp_cap) {
            if (tmp) cudaFree(tmp);
            tmp = nullptr;
            CK(cudaMalloc(&tmp, count * 8));
            tmp_cap = count * 8;
        }
        CK(cudaStreamSynchronize(st));
        g->ptr[rank] = buf;
        if (!g->barrier()) return STEM_E_NCCL;
        PtrSet ps{};
        for (int r = 0; r < world; r++) ps.p[r] = g->ptr[r];
        if (count) sum_buffers_kernel<<<(unsigned)((count + 255) / 256), 256, 0, st>>>(ps, world, count, f64, tmp);
        cudaError_t e = cudaStreamSynchronize(st);
        if (!g->barrier()) return STEM_E_NCCL;   // every rank has read every buffer
        if (e != cudaSuccess) return STEM_E_CUDA;
        CK(cudaMemcpyAsync(buf, tmp, count * 8, cudaMemcpyDeviceToDevice, st));
        CK(cudaStreamSynchronize(st));
        return STEM_OK;
    }
    // the ranks share one device: a peer's buffer is its plain device pointer
    int window(void *const *mine, int nptr, void **peers, cudaStream_t) override {
        g->wptr[rank] = mine;
        if (!g->barrier()) return STEM_E_NCCL;
        for (int r = 0; r < world; r++)
            for (int i = 0; i < nptr; i++) peers[(size_t)r * nptr + i] = g->wptr[r][i];
        if (!g->barrier()) return STEM_E_NCCL;
        return STEM_OK;
    }
    int allgather_host(const uint64_t *mine, size_t count, uint64_t *all, cudaStream_t) override {
        g->h0[rank] = mine;
        if (!g->barrier()) return STEM_E_NCCL;
        for (int r = 0; r < world; r++) memcpy(all + (size_t)r * count, g->h0[r], count * sizeof(uint64_t));
        if (!g->barrier()) return STEM_E_NCCL;
        return STEM_OK;
    }
    int alltoallv(const void *send, const uint64_t *scnt, const uint64_t *sdsp, void *recv, const uint64_t *rcnt,
                  const uint64_t *rdsp, size_t elem, cudaStream_t st) override {
        (void)rcnt;
        CK(cudaStreamSynchronize(st));
        g->ptr[rank] = send;
        g->h0[rank] = scnt;
        g->h1[rank] = sdsp;
        if (!g->barrier()) return STEM_E_NCCL;
        cudaError_t e = cudaSuccess;
        for (int r = 0; r < world && e == cudaSuccess; r++) {
            const uint64_t cnt = g->h0[r][rank];
            if (cnt)
                e = cudaMemcpyAsync((char *)recv + rdsp[r] * elem, (const char *)g->ptr[r] + g->h1[r][rank] * elem,
                                    cnt * elem, cudaMemcpyDeviceToDevice, st);
        }
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
        if (!g->barrier()) return STEM_E_NCCL;   // senders may reuse their buffers
        if (e != cudaSuccess) return STEM_E_CUDA;
        return STEM_OK;
    }
};

// STEMROOT_DIST_P2P=0: the kernel-id exchange by grouped send/recv instead of
// the fused scatter into peer receive windows
static bool dist_p2p() {
    static int v = -1;
    if (v < 0) v = (getenv("STEMROOT_DIST_P2P") && getenv("STEMROOT_DIST_P2P")[0] == '0') ? 0 : 1;
    return v == 1;
}

int sync_stream(Ctx &c) {
    if (c.comm) return c.comm->wait(c.stream);
    CK(cudaStreamSynchronize(c.stream));
    return STEM_OK;
}

// Every rank contributes its local status; all return the first non-OK status
// in rank order (or OK).  Called between stretches of local work and the next
// collective, so no rank is left waiting for a peer that already returned.
int dist_checkpoint(Ctx &c, int status) {
    if (!c.comm) return status;
    const int W = c.comm->world;
    uint64_t mine = (uint64_t)(int64_t)status;
    std::vector<uint64_t> all((size_t)W);
    const int e = c.comm->allgather_host(&mine, 1, all.data(), c.stream);
    if (e != STEM_OK) return e;
    for (int r = 0; r < W; r++)
        if ((int64_t)all[r] != STEM_OK) return (int)(int64_t)all[r];
    return STEM_OK;
}

int comm_rank(const Comm *c) { return c->rank; }
int comm_world(const Comm *c) { return c->world; }
int comm_allgather_host(Ctx &c, const uint64_t *mine, size_t count, uint64_t *all) {
    return c.comm->allgather_host(mine, count, all, c.stream);
}
int comm_alltoallv(Ctx &c, const void *send, const uint64_t *scnt, const uint64_t *sdsp, void *recv,
                   const uint64_t *rcnt, const uint64_t *rdsp, size_t elem) {
    return c.comm->alltoallv(send, scnt, sdsp, recv, rcnt, rdsp, elem, c.stream);
}
int dist_allreduce_u64(Ctx &c, uint64_t *buf, size_t count) { return c.comm->allreduce(buf, count, false, c.stream); }
int dist_allreduce_f64(Ctx &c, double *buf, size_t count) { return c.comm->allreduce(buf, count, true, c.stream); }

// ---------------------------------------------------------------- owner ranges
// bounds[r] = smallest k with sum_{j<k} counts[j] * world >= r * total: contiguous kernel-id
// ranges holding ~total/world rows each (a kernel is never split).
void owner_ranges(const uint64_t *counts, uint32_t K, int world, uint32_t *bounds) {
    u128 total = 0;
    for (uint32_t k = 0; k < K; k++) total += counts[k];
    bounds[0] = 0;
    int r = 1;
    u128 cum = 0;
    for (uint32_t k = 0; k < K && r < world; k++) {
        while (r < world && cum * (u128)world >= (u128)r * total) bounds[r++] = k;
        cum += counts[k];
    }
    while (r < world) bounds[r++] = K;
    bounds[world] = K;
}

// ---------------------------------------------------------------- stable partition by destination
constexpr int kPartThreads = 256, kPartItems = 16;
constexpr uint64_t kPartTile = (uint64_t)kPartThreads * kPartItems;

struct PartArgs {
    const uint32_t *key;            // destination key (kernel id or global row)
    uint64_t key_add;               // key value = key[i] + key_add (key == NULL: key_add + i)
    uint64_t bounds[kMaxWorld + 1]; // dest = #{r in 1..world-1 : bounds[r] <= key}
    int world;
    uint64_t n;
    const uint32_t *in0, *in1;      // payload u32 columns (NULL = skip)
    uint64_t in2_add;               // third u32 column = in2_add + i (the global row), if out2
    const double *inw;              // payload f64 column
    uint32_t *out0, *out1, *out2;
    double *outw;
    // unit mode (kernels larger than a rank's share): the key is the row's unit,
    // kunit[kid] + (its leaf among the kernel's gl_n[kid] value-tree leaves, by t)
    const uint32_t *kunit, *gl_first, *gl_n, *gl_t;
};

__device__ __forceinline__ int part_dest(const PartArgs &a, uint64_t i) {
    uint64_t k = a.key ? (uint64_t)a.key[i] + a.key_add : a.key_add + i;
    if (a.kunit) {
        const uint32_t kid = (uint32_t)k, m = a.gl_n[kid];
        k = a.kunit[kid];
        if (m) k += upper_bound(a.gl_t + a.gl_first[kid], (uint64_t)m, a.in1[i]) - 1;
    }
    int d = 0;
    for (int r = 1; r < a.world; r++) d += a.bounds[r] <= k;
    return d;
}

__global__ void __launch_bounds__(kPartThreads) part_count_kernel(PartArgs a, uint64_t ntiles, uint64_t *cnt) {
    __shared__ uint32_t h[kMaxWorld];
    for (int i = threadIdx.x; i < a.world; i += kPartThreads) h[i] = 0;
    __syncthreads();
    const uint64_t base = blockIdx.x * kPartTile;
    for (int j = 0; j < kPartItems; j++) {
        const uint64_t i = base + (uint64_t)j * kPartThreads + threadIdx.x;
        if (i < a.n) atomicAdd(&h[part_dest(a, i)], 1u);
    }
    __syncthreads();
    for (int d = threadIdx.x; d < a.world; d += kPartThreads) cnt[(uint64_t)d * ntiles + blockIdx.x] = h[d];
}

// Fused exchange: the destinations' receive windows (peer device memory over
// NVLink / NVSwitch, or the other loopback ranks' buffers on this GPU) and, per
// destination d, delta[d] = (my first row in d's window) - (the start of d's
// segment in my partition order).  The scatter stores each row straight into
// its owner's window: no local staging, no send/recv pass.
struct PeerDst {
    uint32_t *kid[kMaxWorld], *t[kMaxWorld], *row[kMaxWorld];
    int64_t delta[kMaxWorld];
};

// stable: element order within each destination is preserved (warp-striped ranking)
template <bool PEER>
__global__ void __launch_bounds__(kPartThreads) part_scatter_kernel(PartArgs a, uint64_t ntiles, const uint64_t *off,
                                                                   const PeerDst *__restrict__ pd) {
    constexpr int NW = kPartThreads / 32;
    __shared__ uint32_t wh[NW][kMaxWorld];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    for (int i = tid; i < NW * kMaxWorld; i += kPartThreads) (&wh[0][0])[i] = 0;
    __syncthreads();
    const uint64_t wbase = blockIdx.x * kPartTile + (uint64_t)w * 32 * kPartItems;
    int dst[kPartItems];
    uint32_t rank[kPartItems];
    for (int j = 0; j < kPartItems; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        const bool valid = i < a.n;
        const uint32_t vmask = __ballot_sync(0xffffffffu, valid);
        dst[j] = 0;
        rank[j] = 0;
        if (valid) {
            const int d = part_dest(a, i);
            const uint32_t peers = __match_any_sync(vmask, d);
            const uint32_t base = wh[w][d];
            const uint32_t below = __popc(peers & ((1u << lane) - 1));
            dst[j] = d;
            rank[j] = base + below;
            __syncwarp(vmask);
            if (below == 0) wh[w][d] = base + __popc(peers);
        }
        __syncwarp();
    }
    __syncthreads();
    if (tid < a.world) {   // exclusive offsets over warps, per destination
        uint32_t run = 0;
        for (int ww = 0; ww < NW; ww++) {
            const uint32_t c = wh[ww][tid];
            wh[ww][tid] = run;
            run += c;
        }
    }
    __syncthreads();
    for (int j = 0; j < kPartItems; j++) {
        const uint64_t i = wbase + (uint64_t)j * 32 + lane;
        if (i >= a.n) continue;
        const int d = dst[j];
        const uint64_t pos = off[(uint64_t)d * ntiles + blockIdx.x] + wh[w][d] + rank[j];
        if (PEER) {
            const uint64_t rp = (uint64_t)((int64_t)pos + pd->delta[d]);
            pd->kid[d][rp] = a.in0[i];
            pd->t[d][rp] = a.in1[i];
            pd->row[d][rp] = (uint32_t)(a.in2_add + i);
            continue;
        }
        if (a.out0) a.out0[pos] = a.in0[i];
        if (a.out1) a.out1[pos] = a.in1[i];
        if (a.out2) a.out2[pos] = (uint32_t)(a.in2_add + i);
        if (a.outw) a.outw[pos] = a.inw[i];
    }
    if (PEER) __threadfence_system();   // the stores are visible to the owners before the barrier
}

__global__ void part_displs_kernel(const uint64_t *off, uint64_t ntiles, int world, uint64_t *displs) {
    const int d = threadIdx.x;
    if (d <= world) displs[d] = off[(uint64_t)d * ntiles];
}

// Runs the partition; host scnt/sdsp get per-destination counts and
// displacements.  pd != NULL: the rows are stored into the owners' windows
// instead (partition_peer), after the counts are known everywhere.
static int partition_count(Ctx &c, PartArgs &a, uint64_t *scnt, uint64_t *sdsp, uint64_t &ntiles) {
    cudaStream_t st = c.stream;
    const int W = a.world;
    ntiles = 0;
    if (a.n == 0) {
        for (int d = 0; d < W; d++) scnt[d] = sdsp[d] = 0;
        return STEM_OK;
    }
    ntiles = (a.n + kPartTile - 1) / kPartTile;
    const uint64_t cells = (uint64_t)W * ntiles;
    CKS(c.ensure(c.part_cnt, c.cap_part_cnt, sizeof(uint64_t) * (cells + 1 + kMaxWorld + 1)));
    CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(cells + 1) + 1) * sizeof(uint64_t)));
    uint64_t *cnt = c.part_cnt, *displs = c.part_cnt + cells + 1;
    part_count_kernel<<<(unsigned)ntiles, kPartThreads, 0, st>>>(a, ntiles, cnt);
    exclusive_scan<uint64_t>([cnt, cells] __device__(uint64_t i) -> uint64_t { return i < cells ? cnt[i] : 0; },
                             [cnt] __device__(uint64_t i, uint64_t pre, uint64_t) { cnt[i] = pre; }, cells + 1,
                             (uint64_t *)c.scan_scratch, &c.scalars->scan_total64, st, &c.launches);
    part_displs_kernel<<<1, kMaxWorld + 1, 0, st>>>(cnt, ntiles, W, displs);
    c.launches += 2;
    CK(cudaGetLastError());
    uint64_t h[kMaxWorld + 1];
    CK(cudaMemcpyAsync(h, displs, sizeof(uint64_t) * (W + 1), cudaMemcpyDeviceToHost, st));
    CKS(sync_stream(c));
    for (int d = 0; d < W; d++) {
        sdsp[d] = h[d];
        scnt[d] = h[d + 1] - h[d];
    }
    return STEM_OK;
}

static int partition_scatter(Ctx &c, PartArgs &a, uint64_t ntiles, const PeerDst *pd_dev) {
    if (!ntiles) return STEM_OK;
    if (pd_dev)
        part_scatter_kernel<true><<<(unsigned)ntiles, kPartThreads, 0, c.stream>>>(a, ntiles, c.part_cnt, pd_dev);
    else
        part_scatter_kernel<false><<<(unsigned)ntiles, kPartThreads, 0, c.stream>>>(a, ntiles, c.part_cnt, nullptr);
    c.launches++;
    CK(cudaGetLastError());
    return STEM_OK;
}

static int partition(Ctx &c, PartArgs &a, uint64_t *scnt, uint64_t *sdsp) {
    uint64_t ntiles = 0;
    CKS(partition_count(c, a, scnt, sdsp, ntiles));
    return partition_scatter(c, a, ntiles, nullptr);
}

// receive layout from everyone's send counts: rcnt[s] = counts s sends to me.
// The allgather also carries every rank's local status (the partition before
// it is local work): all ranks return the first failure in rank order.
static int exchange_counts(Ctx &c, int local_status, const uint64_t *scnt, uint64_t *rcnt, uint64_t *rdsp,
                           uint64_t &total, uint64_t *mystart = nullptr) {
    const int W = c.comm->world, me = c.comm->rank;
    std::vector<uint64_t> mine((size_t)W + 1, 0), all((size_t)W * (W + 1));
    if (local_status == STEM_OK)
        for (int d = 0; d < W; d++) mine[d] = scnt[d];
    mine[W] = (uint64_t)(int64_t)local_status;
    CKS(c.comm->allgather_host(mine.data(), W + 1, all.data(), c.stream));
    for (int r = 0; r < W; r++)
        if ((int64_t)all[(size_t)r * (W + 1) + W] != STEM_OK) return (int)(int64_t)all[(size_t)r * (W + 1) + W];
    total = 0;
    for (int s = 0; s < W; s++) {
        rcnt[s] = all[(size_t)s * (W + 1) + me];
        rdsp[s] = total;
        total += rcnt[s];
    }
    if (mystart)   // where my rows start in destination d's receive order (senders in rank order)
        for (int d = 0; d < W; d++) {
            mystart[d] = 0;
            for (int s = 0; s < me; s++) mystart[d] += all[(size_t)s * (W + 1) + d];
        }
    return STEM_OK;
}

// ---------------------------------------------------------------- metric estimates across ranks
__global__ void __launch_bounds__(256) metric_req_kernel(const uint32_t *rows, const double *w, uint64_t cnt,
                                                         uint64_t row_base, const double *metrics, uint64_t n_local,
                                                         uint32_t nm, double *part) {
    __shared__ double sm[8];
    const uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (uint32_t cc = 0; cc < nm; cc++) {
        double v = 0.0;
        if (s < cnt) v = __dmul_rn(w[s], metrics[(uint64_t)cc * n_local + (rows[s] - row_base)]);
        for (int o = 16; o; o >>= 1) v = __dadd_rn(v, __shfl_xor_sync(0xffffffffu, v, o));
        __syncthreads();
        if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = v;
        __syncthreads();
        if (threadIdx.x == 0) {
            double r = 0.0;
            for (int k = 0; k < 8; k++) r = __dadd_rn(r, sm[k]);
            part[(uint64_t)blockIdx.x * nm + cc] = r;
        }
    }
}

__global__ void cols_sum_kernel(const double *part, uint64_t blocks, uint32_t cols, double *out) {
    const uint32_t cc = threadIdx.x;
    if (cc >= cols) return;
    double r = 0.0;
    for (uint64_t b = 0; b < blocks; b++) r = __dadd_rn(r, part[b * cols + cc]);
    out[cc] = r;
}

// sum over samples of weight * metric[row]: each request goes to the rank holding the row
int dist_metric_sums(Ctx &c, const double *metrics_local, uint32_t nm, uint64_t S, double *out) {
    cudaStream_t st = c.stream;
    const int W = c.comm->world;
    PartArgs a{};
    a.key = c.out_row;
    a.key_add = 0;
    for (int r = 0; r <= W; r++) a.bounds[r] = c.row_bases[r];
    a.world = W;
    a.n = S;
    a.in0 = c.out_row;
    a.inw = c.out_weight;
    uint64_t scnt[kMaxWorld], sdsp[kMaxWorld], rcnt[kMaxWorld], rdsp[kMaxWorld], R = 0;
    const int ls = [&]() -> int {
        CKS(c.ensure(c.xfer_u32[0], c.cap_xfer_u32[0], sizeof(uint32_t) * (S + 1)));
        CKS(c.ensure(c.xfer_f64, c.cap_xfer_f64, sizeof(double) * (S + 1)));
        a.out0 = c.xfer_u32[0];
        a.outw = c.xfer_f64;
        return partition(c, a, scnt, sdsp);
    }();
    CKS(exchange_counts(c, ls, scnt, rcnt, rdsp, R));
    const uint64_t blocks = (R + 255) / 256;
    CKS(dist_checkpoint(c, [&]() -> int {
        CKS(c.ensure(c.xfer_u32[1], c.cap_xfer_u32[1], sizeof(uint32_t) * (R + 1)));
        CKS(c.ensure(c.xfer_f64b, c.cap_xfer_f64b, sizeof(double) * (R + 1)));
        CKS(c.ensure(c.red_part2, c.cap_red2, sizeof(double) * (blocks * nm + nm + 1)));
        return STEM_OK;
    }()));
    CKS(c.comm->alltoallv(c.xfer_u32[0], scnt, sdsp, c.xfer_u32[1], rcnt, rdsp, sizeof(uint32_t), st));
    CKS(c.comm->alltoallv(c.xfer_f64, scnt, sdsp, c.xfer_f64b, rcnt, rdsp, sizeof(double), st));
    CKS(dist_checkpoint(c, [&]() -> int {
        if (R) {
            metric_req_kernel<<<(unsigned)blocks, 256, 0, st>>>(c.xfer_u32[1], c.xfer_f64b, R,
                                                                c.row_bases[c.comm->rank], metrics_local,
                                                                c.n_local_rows, nm, c.red_part2);
            c.launches++;
        }
        cols_sum_kernel<<<1, 64, 0, st>>>(c.red_part2, blocks, nm, out);
        c.launches++;
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    return c.comm->allreduce(out, nm, true, st);
}

// ---------------------------------------------------------------- the distributed plan
__global__ void kid_counts_u64_kernel(const uint32_t *cnt32, uint32_t K, const uint32_t *err, uint64_t *out) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < K) out[i] = cnt32[i];
    if (i == K) out[K] = *err ? 1 : 0;
}

__global__ void sub_kernel_u32(uint32_t *x, uint64_t n, uint32_t v) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) x[i] -= v;
}

__global__ void add_kernel_u32(uint32_t *x, uint64_t n, uint32_t v) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) x[i] += v;
}

// ---------------------------------------------------------------- kernels larger than a rank's share
// A kernel with more than factor * N / P rows (STEMROOT_DIST_GIANT, default
// 1.25; 0 disables) would overload the rank owning it.  Its ROOT tree is built
// instead from its value histogram (root.cu root_values: the decisions depend
// only on the multiset of times, so the tree is the row tree): every rank
// histograms its rows of the kernel, the histograms are merged on every rank,
// every rank builds the same value tree, and the kernel's LEAVES become units of
// ownership next to the whole ordinary kernels.  Units are dealt to ranks in
// (kernel, value) order, so the gathered plan is still in (kernel, ordinal)
// order; a rank keeps the leaves it owns fixed (no ROOT on them) and numbers
// them from the kernel's global ordinal.  Used with the exact 2-means split and
// the global or per-leaf scopes (the Lloyd rules and the per-kernel solve keep
// whole kernels).
struct GiantPlan {
    bool on = false;
    std::vector<uint32_t> ubounds;          // [W + 1] first unit of each rank
    uint32_t kb = 0, ke = 0;                // my kernel range [kb, ke)
    uint32_t *kunit = nullptr, *gl_first = nullptr, *gl_n = nullptr, *gl_t = nullptr;   // device tables
    uint8_t *fixed = nullptr;               // device [ke - kb]
    uint32_t *ord_off = nullptr;            // device [ke - kb]
    uint32_t *cuts = nullptr;               // device pairs (local kernel, rows from the local group start)
    uint64_t ncuts = 0;
};

static double giant_factor() {
    static double v = -1.0;
    if (v < 0.0) {
        const char *e = getenv("STEMROOT_DIST_GIANT");
        v = e ? atof(e) : 1.25;
        if (!(v >= 0.0)) v = 1.25;
    }
    return v;
}

__global__ void gi_group_kernel(const uint32_t *goff, uint32_t G, uint64_t m, uint32_t *grp) {
    const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < m) grp[i] = (uint32_t)(upper_bound(goff, (uint64_t)G + 1, (uint32_t)i) - 1);
}

__global__ void gi_counts_kernel(const uint32_t *start, uint64_t nrec, uint64_t total, uint32_t *cnt) {
    const uint64_t r = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r < nrec) cnt[r] = (uint32_t)((r + 1 < nrec ? start[r + 1] : total) - start[r]);
}

__global__ void gi_vcnt_kernel(const uint32_t *vstart, uint64_t D, uint64_t total, const uint64_t *cp, uint64_t *vcnt) {
    const uint64_t u = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (u < D) vcnt[u] = cp[u + 1 < D ? vstart[u + 1] : total] - cp[vstart[u]];
}

__global__ void gi_goffv_kernel(const uint32_t *goff, uint32_t G, const uint32_t *vstart, uint64_t D, uint32_t *goffv) {
    const uint32_t g = blockIdx.x * blockDim.x + threadIdx.x;
    if (g <= G) goffv[g] = (uint32_t)lower_bound(vstart, D, goff[g]);
}

template <class T>
static int up(Ctx &c, T *dst, const std::vector<T> &v) {
    if (!v.empty()) CK(cudaMemcpyAsync(dst, v.data(), sizeof(T) * v.size(), cudaMemcpyHostToDevice, c.stream));
    return STEM_OK;
}

// Builds the value trees of the giant kernels and the unit owner map.  Collective.
static int giant_plan(Ctx &c, Comm &comm, const uint32_t *kid, const uint32_t *t, uint64_t n, uint32_t K,
                      const std::vector<uint64_t> &gcnt, const std::vector<uint32_t> &giant, double eps, double z,
                      int clamp, GiantPlan &gp) {
    cudaStream_t st = c.stream;
    const int W = comm.world, me = comm.rank;
    const uint32_t G = (uint32_t)giant.size();
    const double k2 = (z / eps) * (z / eps);
    std::vector<uint32_t> gidx_h(K, 0xFFFFFFFFu);
    for (uint32_t g = 0; g < G; g++) gidx_h[giant[g]] = g;
    // 1. this rank's rows of the giant kernels, sorted by (giant, t), run-length encoded
    uint64_t ng = 0, nrec = 0;
    uint32_t *rec = nullptr;   // [3][nrec]: giant, t, count
    CKS(dist_checkpoint(c, [&]() -> int {
        CKS(c.ensure(c.gi_tab, c.cap_gi_tab, sizeof(uint32_t) * ((uint64_t)K + 1)));
        uint32_t *gidx = (uint32_t *)c.gi_tab;
        CKS(up(c, gidx, gidx_h));
        for (int i = 0; i < 2; i++) CKS(c.ensure(c.xfer_u32[i], c.cap_xfer_u32[i], sizeof(uint32_t) * (n + 1)));
        CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(n + 1) + 1) * sizeof(uint64_t)));
        uint32_t *ga = c.xfer_u32[0], *ta = c.xfer_u32[1];
        exclusive_scan<uint64_t>(
            [kid, gidx] __device__(uint64_t i) -> uint64_t { return gidx[kid[i]] != 0xFFFFFFFFu ? 1ull : 0ull; },
            [kid, t, gidx, ga, ta] __device__(uint64_t i, uint64_t pre, uint64_t v) {
                if (v) { ga[pre] = gidx[kid[i]]; ta[pre] = t[i]; }
            },
            n, (uint64_t *)c.scan_scratch, &c.scalars->scan_total64, st, &c.launches);
        CK(cudaMemcpyAsync(&ng, &c.scalars->scan_total64, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        CKS(sync_stream(c));
        CKS(c.ensure(c.gi_rec, c.cap_gi_rec, sizeof(uint32_t) * 4 * (ng + 1)));
        rec = (uint32_t *)c.gi_rec;
        if (!ng) return STEM_OK;
        CKS(c.ensure_all(ng, G, 0));
        CKS(sort_trace(c, ga, ta, nullptr, ng, G, false));
        uint32_t *grp = rec + 3 * (ng + 1);   // scratch: giant of each sorted position
        gi_group_kernel<<<(unsigned)((ng + 255) / 256), 256, 0, st>>>(c.goff, G, ng, grp);
        const uint32_t *ts = c.t_sorted;
        uint32_t *rg = rec, *rt = rec + (ng + 1), *rs = rec + 2 * (ng + 1);
        exclusive_scan<uint64_t>(
            [ts, grp] __device__(uint64_t i) -> uint64_t {
                return (i == 0 || grp[i] != grp[i - 1] || ts[i] != ts[i - 1]) ? 1ull : 0ull;
            },
            [ts, grp, rg, rt, rs] __device__(uint64_t i, uint64_t pre, uint64_t v) {
                if (v) { rg[pre] = grp[i]; rt[pre] = ts[i]; rs[pre] = (uint32_t)i; }
            },
            ng, (uint64_t *)c.scan_scratch, &c.scalars->scan_total64, st, &c.launches);
        CK(cudaMemcpyAsync(&nrec, &c.scalars->scan_total64, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        CKS(sync_stream(c));
        gi_counts_kernel<<<(unsigned)((nrec + 255) / 256), 256, 0, st>>>(rs, nrec, ng, grp);
        CK(cudaMemcpyAsync(rs, grp, sizeof(uint32_t) * nrec, cudaMemcpyDeviceToDevice, st));   // starts -> counts
        c.launches += 2;
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    // 2. every rank's records, on every rank (rank order)
    std::vector<uint64_t> cnts((size_t)W);
    CKS(comm.allgather_host(&nrec, 1, cnts.data(), st));
    uint64_t Rall = 0;
    std::vector<uint64_t> scnt(W, nrec), sdsp(W, 0), rcnt(W), rdsp(W);
    for (int r = 0; r < W; r++) { rcnt[r] = cnts[r]; rdsp[r] = Rall; Rall += cnts[r]; }
    uint32_t *all = nullptr;
    CKS(dist_checkpoint(c, [&]() -> int {
        CKS(c.ensure(c.gi_all, c.cap_gi_all, sizeof(uint32_t) * 3 * (Rall + 1)));
        all = (uint32_t *)c.gi_all;
        return STEM_OK;
    }()));
    const uint32_t *rsrc = (const uint32_t *)c.gi_rec;
    for (int f = 0; f < 3; f++)
        CKS(comm.alltoallv(rsrc + f * (ng + 1), scnt.data(), sdsp.data(), all + f * (Rall + 1), rcnt.data(),
                           rdsp.data(), sizeof(uint32_t), st));
    CKS(sync_stream(c));
    // 3. merged histogram (identical on every rank), the value trees, the leaves
    std::vector<uint32_t> l_g, l_t;
    std::vector<uint64_t> l_rows;
    CKS(dist_checkpoint(c, [&]() -> int {
        if (!Rall) return STEM_OK;
        uint32_t *ag = all, *at = all + (Rall + 1), *ac = all + 2 * (Rall + 1);
        CKS(c.ensure_all(Rall, G, 0));
        CKS(sort_trace(c, ag, at, ac, Rall, G, false));   // payload = the counts
        const uint32_t *ts = c.t_sorted, *cs = c.row_sorted, *goff = c.goff;
        CKS(c.ensure(c.scan_scratch, c.cap_scan, (scan_tiles(Rall + 1) + 1) * sizeof(uint64_t)));
        const uint64_t R2 = (Rall + 2 + 1) & ~1ull, G2 = (G + 2 + 1) & ~1ull;   // even: 8-byte aligned after
        CKS(c.ensure(c.gi_val, c.cap_gi_val, sizeof(uint32_t) * (3 * R2 + G2) + sizeof(uint64_t) * 2 * R2 + R2));
        uint32_t *grp = (uint32_t *)c.gi_val, *vt = grp + R2, *vstart = vt + R2, *goffv = vstart + R2;
        uint64_t *cp = (uint64_t *)(goffv + G2), *vcnt = cp + R2;
        uint8_t *vflag = (uint8_t *)(vcnt + R2);
        gi_group_kernel<<<(unsigned)((Rall + 255) / 256), 256, 0, st>>>(goff, G, Rall, grp);
        exclusive_scan<uint64_t>([cs] __device__(uint64_t i) -> uint64_t { return cs[i]; },
                                 [cp] __device__(uint64_t i, uint64_t pre, uint64_t) { cp[i] = pre; }, Rall,
                                 (uint64_t *)c.scan_scratch, &c.scalars->scan_total64, st, &c.launches);
        uint64_t D = 0;
        exclusive_scan<uint64_t>(
            [ts, grp] __device__(uint64_t i) -> uint64_t {
                return (i == 0 || grp[i] != grp[i - 1] || ts[i] != ts[i - 1]) ? 1ull : 0ull;
            },
            [ts, vt, vstart] __device__(uint64_t i, uint64_t pre, uint64_t v) {
                if (v) { vt[pre] = ts[i]; vstart[pre] = (uint32_t)i; }
            },
            Rall, (uint64_t *)c.scan_scratch, &c.scalars->scan_total64b, st, &c.launches);
        uint64_t tot_rows = 0;
        CK(cudaMemcpyAsync(&D, &c.scalars->scan_total64b, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(&tot_rows, &c.scalars->scan_total64, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        CKS(sync_stream(c));
        CK(cudaMemcpyAsync(cp + Rall, &tot_rows, sizeof(uint64_t), cudaMemcpyHostToDevice, st));
        gi_vcnt_kernel<<<(unsigned)((D + 255) / 256), 256, 0, st>>>(vstart, D, Rall, cp, vcnt);
        gi_goffv_kernel<<<(unsigned)((G + 256) / 256), 256, 0, st>>>(goff, G, vstart, D, goffv);
        c.launches += 3;
        CK(cudaGetLastError());
        CKS(root_values(c, vt, vcnt, goffv, G, D, eps, z, k2, clamp, vflag));
        // leaves: value starts with vflag set, their giant, lowest t and rows (from the prefix counts)
        std::vector<uint8_t> vf(D);
        std::vector<uint32_t> vt_h(D), goffv_h(G + 1);
        std::vector<uint64_t> vcnt_h(D);
        CK(cudaMemcpyAsync(vf.data(), vflag, D, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(vt_h.data(), vt, sizeof(uint32_t) * D, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(vcnt_h.data(), vcnt, sizeof(uint64_t) * D, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(goffv_h.data(), goffv, sizeof(uint32_t) * (G + 1), cudaMemcpyDeviceToHost, st));
        CKS(sync_stream(c));
        for (uint32_t g = 0; g < G; g++)   // (host bookkeeping of the tree's leaves: list building only)
            for (uint32_t u = goffv_h[g]; u < goffv_h[g + 1]; u++) {
                if (vf[u] || u == goffv_h[g]) {
                    l_g.push_back(g);
                    l_t.push_back(vt_h[u]);
                    l_rows.push_back(0);
                }
                l_rows.back() += vcnt_h[u];
            }
        return STEM_OK;
    }()));
    // 4. units in (kernel, value) order and the owner map over them
    std::vector<uint64_t> urows;
    std::vector<uint32_t> ukid, uleaf, kunit_h(K + 1), gl_first_h(K, 0), gl_n_h(K, 0), gl_t_h;
    {
        std::vector<uint32_t> gfirst(G + 1, 0);
        for (size_t i = 0; i < l_g.size(); i++) gfirst[l_g[i] + 1]++;
        for (uint32_t g = 0; g < G; g++) gfirst[g + 1] += gfirst[g];
        for (uint32_t k = 0; k < K; k++) {
            kunit_h[k] = (uint32_t)urows.size();
            const uint32_t g = gidx_h[k];
            if (g == 0xFFFFFFFFu || gfirst[g + 1] == gfirst[g]) {
                urows.push_back(gcnt[k]);
                ukid.push_back(k);
                uleaf.push_back(0);
                continue;
            }
            gl_first_h[k] = (uint32_t)gl_t_h.size();
            gl_n_h[k] = gfirst[g + 1] - gfirst[g];
            for (uint32_t j = gfirst[g]; j < gfirst[g + 1]; j++) {
                urows.push_back(l_rows[j]);
                ukid.push_back(k);
                uleaf.push_back(j - gfirst[g]);
                gl_t_h.push_back(l_t[j]);
            }
        }
        kunit_h[K] = (uint32_t)urows.size();
    }
    const uint32_t U = (uint32_t)urows.size();
    gp.ubounds.assign(W + 1, 0);
    owner_ranges(urows.data(), U, W, gp.ubounds.data());
    const uint32_t u0 = gp.ubounds[me], u1 = gp.ubounds[me + 1];
    gp.kb = u0 < u1 ? ukid[u0] : 0;
    gp.ke = u0 < u1 ? ukid[u1 - 1] + 1 : 0;
    const uint32_t KL = gp.ke - gp.kb;
    std::vector<uint8_t> fixed_h(KL + 1, 0);
    std::vector<uint32_t> ord_h(KL + 1, 0), cuts_h;
    for (uint32_t u = u0; u < u1; u++) {
        const uint32_t kl = ukid[u] - gp.kb;
        if (gl_n_h[ukid[u]] == 0) continue;
        if (!fixed_h[kl]) {   // the first leaf of this kernel on this rank
            fixed_h[kl] = 1;
            ord_h[kl] = uleaf[u];
            continue;
        }
        uint64_t rel = 0;     // rows of this kernel's earlier local leaves
        for (uint32_t v = u; v-- > u0 && ukid[v] == ukid[u];) rel += urows[v];
        cuts_h.push_back(kl);
        cuts_h.push_back((uint32_t)rel);
    }
    gp.ncuts = cuts_h.size() / 2;
    CKS(dist_checkpoint(c, [&]() -> int {
        const size_t words = (size_t)3 * (K + 1) + gl_t_h.size() + 2 * (KL + 1) + cuts_h.size() + 8;
        CKS(c.ensure(c.gi_tab, c.cap_gi_tab, sizeof(uint32_t) * words));
        uint32_t *w = (uint32_t *)c.gi_tab;
        gp.kunit = w; w += K + 1;
        gp.gl_first = w; w += K + 1;
        gp.gl_n = w; w += K + 1;
        gp.gl_t = w; w += gl_t_h.size() + 1;
        gp.ord_off = w; w += KL + 1;
        gp.cuts = w; w += cuts_h.size() + 1;
        gp.fixed = (uint8_t *)w;
        CKS(up(c, gp.kunit, kunit_h));
        gl_first_h.push_back(0);
        gl_n_h.push_back(0);
        CKS(up(c, gp.gl_first, gl_first_h));
        CKS(up(c, gp.gl_n, gl_n_h));
        CKS(up(c, gp.gl_t, gl_t_h));
        CKS(up(c, gp.ord_off, ord_h));
        CKS(up(c, gp.cuts, cuts_h));
        CKS(up(c, gp.fixed, fixed_h));
        return sync_stream(c);   // the host vectors are this frame's
    }()));
    gp.on = true;
    return STEM_OK;
}

// local_status: the rank's own argument checks (stem_root_plan_dist), agreed
// across ranks first.  Every later stretch of local work ends in a checkpoint
// (or in exchange_counts, which carries the status) before the next
// collective, so all ranks return the same status together.
int run_plan_dist(Ctx &c, Comm &comm, const stem_trace *tr, uint64_t row_base, double eps, double conf,
                  const stem_opts &o, int local_status) {
    const int W = comm.world, me = comm.rank;
    const uint64_t n = tr->n;
    const uint32_t K = tr->n_kernels, nm = tr->n_metrics;
    cudaStream_t st = c.stream;
    const uint32_t *kid = tr->kernel_id, *t = tr->exec_ns;
    const double *met = tr->metrics;
    (void)conf;
    // ---- arguments, input copy-in, histogram buffers
    CKS(dist_checkpoint(c, [&]() -> int {
        CKS(local_status);
        if (tr->device < 0 && n) {   // host shard: copy in on the stream
            CKS(c.ensure(c.in_kid, c.cap_in_kid, sizeof(uint32_t) * n));
            CKS(c.ensure(c.in_t, c.cap_in_t, sizeof(uint32_t) * n));
            CK(cudaMemcpyAsync(c.in_kid, kid, sizeof(uint32_t) * n, cudaMemcpyHostToDevice, st));
            CK(cudaMemcpyAsync(c.in_t, t, sizeof(uint32_t) * n, cudaMemcpyHostToDevice, st));
            kid = c.in_kid;
            t = c.in_t;
            if (nm) {
                CKS(c.ensure(c.in_met, c.cap_in_met, sizeof(double) * n * nm));
                CK(cudaMemcpyAsync(c.in_met, met, sizeof(double) * n * nm, cudaMemcpyHostToDevice, st));
                met = c.in_met;
            }
        }
        CKS(c.ensure(c.kid_count, c.cap_kc, sizeof(uint32_t) * ((uint64_t)K + 1)));
        CKS(c.ensure(c.dist_cnt, c.cap_dist_cnt, sizeof(uint64_t) * ((uint64_t)K + 2)));
        CKS(c.ensure(c.scalars, c.cap_scalars, sizeof(DevScalars)));
        CKS(c.ensure(c.kid_max, c.cap_kmax, sizeof(uint32_t) * ((uint64_t)K + 1)));
        CKS(c.ensure(c.hist, c.cap_hist, sizeof(uint64_t) * 9 * 256));
        return STEM_OK;
    }()));
    // row shards of every rank (metric requests are routed by row); the checks
    // run on the same gathered data everywhere, so every rank agrees
    {
        uint64_t mine[2] = {row_base, n};
        std::vector<uint64_t> all(2 * (size_t)W);
        CKS(comm.allgather_host(mine, 2, all.data(), st));
        for (int r = 0; r < W; r++) {
            c.row_bases[r] = all[2 * r];
            if (r > 0 && all[2 * r] != all[2 * (r - 1)] + all[2 * (r - 1) + 1]) return STEM_E_INVAL;   // contiguous
        }
        c.row_bases[W] = all[2 * (W - 1)] + all[2 * (W - 1) + 1];
        if (c.row_bases[W] >= (1ull << 32)) return STEM_E_RANGE;
        c.n_local_rows = n;
    }
    // 1. global kernel histogram (+ range errors) -> owner ranges
    const int tk_x = c.stage_begin("dist_exchange");
    CKS(dist_checkpoint(c, [&]() -> int {
        CK(cudaMemsetAsync(c.scalars, 0, sizeof(DevScalars), st));
        CK(cudaMemsetAsync(c.kid_count, 0, sizeof(uint32_t) * ((uint64_t)K + 1), st));
        if (n) CKS(histogram_kernels(c, kid, t, n, K, nullptr));
        kid_counts_u64_kernel<<<(unsigned)((K + 256) / 256), 256, 0, st>>>(c.kid_count, K, &c.scalars->err,
                                                                           c.dist_cnt);
        c.launches++;
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    CKS(comm.allreduce(c.dist_cnt, (size_t)K + 1, false, st));
    std::vector<uint64_t> gcnt((size_t)K + 1);
    CK(cudaMemcpyAsync(gcnt.data(), c.dist_cnt, sizeof(uint64_t) * ((uint64_t)K + 1), cudaMemcpyDeviceToHost, st));
    CKS(sync_stream(c));
    if (gcnt[K]) return STEM_E_RANGE;   // the same reduced flag on every rank
    std::vector<uint32_t> bounds(W + 1);
    owner_ranges(gcnt.data(), K, W, bounds.data());
    uint32_t kb = bounds[me], ke = bounds[me + 1];
    // kernels larger than a rank's share: value trees and unit ownership (identical decision on every rank)
    GiantPlan gp;
    {
        std::vector<uint32_t> giant;
        uint64_t N = 0;
        for (uint32_t k = 0; k < K; k++) N += gcnt[k];
        const double f = giant_factor();
        if (W > 1 && f > 0.0 && o.root && o.split == 0 && o.scope != 1)
            for (uint32_t k = 0; k < K; k++)
                if ((double)gcnt[k] * W > f * (double)N) giant.push_back(k);
        if (!giant.empty()) {
            CKS(giant_plan(c, comm, kid, t, n, K, gcnt, giant, eps, c.z, o.clamp_in_split ? 1 : 0, gp));
            kb = gp.kb;
            ke = gp.ke;
        }
    }
    // 2. all-to-all keyed on kernel id: (kernel_id, t, global row) to the owner of the kernel
    PartArgs pa{};
    pa.key = kid;
    for (int r = 0; r <= W; r++) pa.bounds[r] = gp.on ? gp.ubounds[r] : bounds[r];
    if (gp.on) {
        pa.kunit = gp.kunit;
        pa.gl_first = gp.gl_first;
        pa.gl_n = gp.gl_n;
        pa.gl_t = gp.gl_t;
    }
    pa.world = W;
    pa.n = n;
    pa.in0 = kid;
    pa.in1 = t;
    pa.in2_add = row_base;
    uint64_t scnt[kMaxWorld], sdsp[kMaxWorld], rcnt[kMaxWorld], rdsp[kMaxWorld], mystart[kMaxWorld], R = 0;
    uint64_t ntiles = 0;
    const bool p2p = dist_p2p();
    auto stage_rows = [&]() -> int {   // the send/recv path: rows staged by destination locally
        for (int i = 0; i < 3; i++) CKS(c.ensure(c.xfer_u32[i], c.cap_xfer_u32[i], sizeof(uint32_t) * (n + 1)));
        pa.out0 = c.xfer_u32[0];
        pa.out1 = c.xfer_u32[1];
        pa.out2 = c.xfer_u32[2];
        return partition_scatter(c, pa, ntiles, nullptr);
    };
    const int ls = [&]() -> int {
        CKS(partition_count(c, pa, scnt, sdsp, ntiles));
        return p2p ? STEM_OK : stage_rows();
    }();
    CKS(exchange_counts(c, ls, scnt, rcnt, rdsp, R, mystart));
    CKS(dist_checkpoint(c, [&]() -> int {
        if (R >= (1ull << 32)) return STEM_E_RANGE;
        for (int i = 0; i < 3; i++) CKS(c.ensure(c.recv_u32[i], c.cap_recv_u32[i], sizeof(uint32_t) * (R + 1)));
        return STEM_OK;
    }()));
    bool fused = false;
    if (p2p) {   // the fused exchange: every row stored straight into its owner's receive window
        void *mine[3] = {c.recv_u32[0], c.recv_u32[1], c.recv_u32[2]};
        std::vector<void *> peers(3 * (size_t)W);
        const int ws = comm.window(mine, 3, peers.data(), st);
        if (ws == STEM_E_NCCL) return ws;
        if (ws == STEM_OK) {   // (STEM_E_CUDA, agreed by every rank: no peer access, use send/recv)
            CKS(dist_checkpoint(c, [&]() -> int {
                PeerDst h{};
                for (int d = 0; d < W; d++) {
                    h.kid[d] = (uint32_t *)peers[3 * d];
                    h.t[d] = (uint32_t *)peers[3 * d + 1];
                    h.row[d] = (uint32_t *)peers[3 * d + 2];
                    h.delta[d] = (int64_t)mystart[d] - (int64_t)sdsp[d];
                }
                CKS(c.ensure(c.peer_dst, c.cap_peer_dst, sizeof(PeerDst)));
                CK(cudaMemcpyAsync(c.peer_dst, &h, sizeof(PeerDst), cudaMemcpyHostToDevice, st));
                CKS(partition_scatter(c, pa, ntiles, (const PeerDst *)c.peer_dst));
                return sync_stream(c);   // h lives on this stack frame until the copy is done
            }()));   // every rank's stores have landed once all ranks pass this point
            fused = true;
        }
    }
    if (!fused) {
        if (p2p) CKS(dist_checkpoint(c, stage_rows()));
        for (int i = 0; i < 3; i++)
            CKS(comm.alltoallv(c.xfer_u32[i], scnt, sdsp, c.recv_u32[i], rcnt, rdsp, sizeof(uint32_t), st));
    }
    c.stats.fused_exchange = fused ? 1u : 0u;
    CKS(sync_stream(c));   // the exchange is complete (or failed) before the local pipeline
    c.stage_end(tk_x, (fused ? 8 + 12 : 8 + 24) * n + (fused ? 0 : 12) * R);
    // 3. the local pipeline on my kernel range (kernel ids rebased to 0)
    const uint32_t KL = ke - kb;
    c.kid_base = kb;
    if (gp.on) {   // this rank's leaves of split kernels are given: no ROOT on them, ordinals from the tree
        c.fixed_kernel = gp.fixed;
        c.fixed_cuts = gp.cuts;
        c.n_fixed_cuts = gp.ncuts;
        c.ord_off = gp.ord_off;
    }
    struct Unfix {
        Ctx &c;
        ~Unfix() { c.fixed_kernel = nullptr; c.fixed_cuts = nullptr; c.n_fixed_cuts = 0; c.ord_off = nullptr; }
    } unfix{c};
    CKS(dist_checkpoint(c, [&]() -> int {
        if (!R) return STEM_OK;
        sub_kernel_u32<<<(unsigned)((R + 255) / 256), 256, 0, st>>>(c.recv_u32[0], R, kb);
        c.launches++;
        CKS(c.ensure_all(R, KL, nm));
        CKS(sort_trace(c, c.recv_u32[0], c.recv_u32[1], c.recv_u32[2], R, KL, !o.census_cap));
        CKS(prefix_moments(c, R));
        if (o.root && o.split == 3) {
            CKS(root_levels_kmeans(c, R, KL, eps, c.z, c.z / eps * (c.z / eps), o.clamp_in_split ? 1 : 0,
                                   (uint32_t)o.kmeans_k));
        } else if (o.root) {
            CKS(root_levels(c, R, KL, eps, c.z, c.z / eps * (c.z / eps), o.clamp_in_split ? 1 : 0, o.split,
                            o.seed));
        } else {
            CKS(stem_only_leaves(c, R, KL));
        }
        return STEM_OK;
    }()));
    const double q = c.z / eps;
    CKS(leaves_and_plan(c, R, KL, met, nm, eps, c.z, q * q, o));
    c.have_mbounds = false;
    if (o.metric_bounds && nm) {   // every rank's leaves gathered; each rank reads its home rows' metrics
        const int tk_mb = c.stage_begin("metric_bounds");
        CKS(metric_bounds_dist(c, c.n_leaves, R, K, kid, t, met, n, nm, c.z));
        c.stage_end(tk_mb, (16 + 16 * (uint64_t)nm) * n);
        c.have_mbounds = true;
    }
    // 4. gather the plan on rank 0, canonical order = rank order (kernel ranges ascend)
    uint64_t mine[2] = {c.n_leaves, c.n_samples};
    std::vector<uint64_t> all(2 * (size_t)W);
    CKS(comm.allgather_host(mine, 2, all.data(), st));
    uint64_t Lg = 0, Sg = 0, Loff = 0;
    for (int r = 0; r < W; r++) {
        if (r == me) Loff = Lg;
        Lg += all[2 * r];
        Sg += all[2 * r + 1];
    }
    std::vector<uint64_t> s_c(W, 0), s_d(W, 0), r_c(W, 0), r_d(W, 0);
    std::vector<uint64_t> rc_all[2];
    for (int which = 0; which < 2; which++) {
        rc_all[which].assign(2 * (size_t)W, 0);
        uint64_t off = 0;
        for (int r = 0; r < W; r++) {
            rc_all[which][r] = all[2 * r + which];
            rc_all[which][W + r] = off;
            off += all[2 * r + which];
        }
    }
    CKS(dist_checkpoint(c, [&]() -> int {
        if (c.n_samples && Loff) {
            add_kernel_u32<<<(unsigned)((c.n_samples + 255) / 256), 256, 0, st>>>(c.out_cluster, c.n_samples,
                                                                                 (uint32_t)Loff);
            c.launches++;
        }
        if (me == 0) {
            CKS(c.ensure(c.g_clusters, c.cap_g_clusters, sizeof(stem_cluster) * (Lg + 1)));
            CKS(c.ensure(c.g_row, c.cap_g_row, sizeof(uint32_t) * (Sg + 1)));
            CKS(c.ensure(c.g_cluster, c.cap_g_cluster, sizeof(uint32_t) * (Sg + 1)));
            CKS(c.ensure(c.g_weight, c.cap_g_weight, sizeof(double) * (Sg + 1)));
        }
        CK(cudaGetLastError());
        return STEM_OK;
    }()));
    auto gather = [&](void *src, void *dst, size_t elem, int which) -> int {
        s_c[0] = all[2 * me + which];
        if (me == 0)
            for (int r = 0; r < W; r++) {
                r_c[r] = rc_all[which][r];
                r_d[r] = rc_all[which][W + r];
            }
        return comm.alltoallv(src, s_c.data(), s_d.data(), dst, r_c.data(), r_d.data(), elem, st);
    };
    CKS(gather(c.out_clusters, c.g_clusters, sizeof(stem_cluster), 0));
    CKS(gather(c.out_row, c.g_row, sizeof(uint32_t), 1));
    CKS(gather(c.out_cluster, c.g_cluster, sizeof(uint32_t), 1));
    CKS(gather(c.out_weight, c.g_weight, sizeof(double), 1));
    CKS(sync_stream(c));
    if (me == 0) {   // the global plan becomes this ctx's output
        std::swap(c.out_clusters, *(stem_cluster **)&c.g_clusters);
        std::swap(c.cap_out_cl, c.cap_g_clusters);
        std::swap(c.out_row, *(uint32_t **)&c.g_row);
        std::swap(c.cap_out_row, c.cap_g_row);
        std::swap(c.out_cluster, *(uint32_t **)&c.g_cluster);
        std::swap(c.cap_out_cluster, c.cap_g_cluster);
        std::swap(c.out_weight, *(double **)&c.g_weight);
        std::swap(c.cap_out_weight, c.cap_g_weight);
        c.n_leaves = Lg;
        c.n_samples = Sg;
    }
    // other ranks keep their own part (its clusters, its samples with global
    // cluster indices): stem_ctx_device_plan then describes exactly the buffers it holds
    c.stats.n_clusters = Lg;
    c.stats.n_samples = Sg;
    c.stats.owned_rows = R;
    c.stats.world = (uint32_t)W;
    return STEM_OK;
}

}  // namespace sr

// ---------------------------------------------------------------- C ABI
struct stem_comm {
    std::unique_ptr<sr::Comm> c;
};

extern "C" {

int stem_comm_nccl_unique_id(void *id_out) {
    if (!id_out) return STEM_E_INVAL;
    if (!sr::nccl().ok) return STEM_E_NCCL;
    ncclUniqueId id;
    if (sr::nccl().getUniqueId(&id) != ncclSuccess) return STEM_E_NCCL;
    memcpy(id_out, &id, sizeof(id));
    return STEM_OK;
}

int stem_comm_init_nccl(const void *id, int rank, int world, int device, stem_comm **out) {
    if (!out) return STEM_E_INVAL;
    *out = nullptr;
    if (!id || world < 1 || world > sr::kMaxWorld || rank < 0 || rank >= world || device < 0) return STEM_E_INVAL;
    if (!sr::nccl().ok) return STEM_E_NCCL;
    if (cudaSetDevice(device) != cudaSuccess) return STEM_E_CUDA;
    auto nc = std::make_unique<sr::NcclComm>();
    nc->rank = rank;
    nc->world = world;
    nc->device = device;
    ncclUniqueId uid;
    memcpy(&uid, id, sizeof(uid));
    if (sr::nccl().commInitRank(&nc->comm, world, uid, rank) != ncclSuccess) {
        nc->comm = nullptr;
        return STEM_E_NCCL;
    }
    stem_comm *x = new (std::nothrow) stem_comm();
    if (!x) return STEM_E_NOMEM;
    x->c = std::move(nc);
    *out = x;
    return STEM_OK;
}

int stem_comm_init_loopback(int world, int device, stem_comm **comms) {
    if (!comms || world < 1 || world > sr::kMaxWorld || device < 0) return STEM_E_INVAL;
    auto g = std::make_shared<sr::LoopGroup>(world);
    for (int r = 0; r < world; r++) {
        auto lc = std::make_unique<sr::LoopComm>();
        lc->rank = r;
        lc->world = world;
        lc->device = device;
        lc->g = g;
        comms[r] = new stem_comm();
        comms[r]->c = std::move(lc);
    }
    return STEM_OK;
}

void stem_comm_destroy(stem_comm *c) { delete c; }

int stem_owner_ranges(const uint64_t *counts, uint32_t n_kernels, int world, uint32_t *bounds) {
    if (!counts || !bounds || world < 1 || world > sr::kMaxWorld || n_kernels == 0) return STEM_E_INVAL;
    sr::owner_ranges(counts, n_kernels, world, bounds);
    return STEM_OK;
}

}  // extern "C"

// the dist entry point lives with the ctx in capi.cu; this accessor bridges the opaque handle
sr::Comm *stem_comm_impl(stem_comm *c) { return c ? c->c.get() : nullptr; }
