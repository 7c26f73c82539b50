// transport.cu — NCCL and in-process group implementations of the exchange seam (transport.h).
#include <chrono>
#include <cstring>
#include <new>

#include <nccl.h>

#include "dense_dev.cuh"
#include "internal.h"
#include "kernels.h"
#include "transport.h"

// ---------------------------------------------------------------------------------------
// NCCL (one process per GPU; P:45 block rows over NVLink / NVSwitch)
// ---------------------------------------------------------------------------------------
namespace {

struct NcclTransport final : Transport {
    ncclComm_t comm = nullptr;
    ~NcclTransport() override {
        if (comm) ncclCommDestroy(comm);
    }
    int allreduce_sum(double* buf, size_t cnt, cudaStream_t st) override {
        if (cnt == 0) return CAGMRES_OK;
        return ncclAllReduce(buf, buf, cnt, ncclDouble, ncclSum, comm, st) == ncclSuccess ? CAGMRES_OK
                                                                                          : CAGMRES_ENCCL;
    }
    int allgather(const void* send, void* recv, size_t bytes, cudaStream_t st) override {
        return ncclAllGather(send, recv, bytes, ncclChar, comm, st) == ncclSuccess ? CAGMRES_OK : CAGMRES_ENCCL;
    }
    int exchange(const std::vector<Msg>& sends, const std::vector<Msg>& recvs, cudaStream_t st) override {
        if (ncclGroupStart() != ncclSuccess) return CAGMRES_ENCCL;
        int bad = 0;
        for (const Msg& m : sends)
            if (m.bytes) bad |= ncclSend(m.ptr, m.bytes, ncclChar, m.peer, comm, st) != ncclSuccess;
        for (const Msg& m : recvs)
            if (m.bytes) bad |= ncclRecv(m.ptr, m.bytes, ncclChar, m.peer, comm, st) != ncclSuccess;
        bad |= ncclGroupEnd() != ncclSuccess;
        return bad ? CAGMRES_ENCCL : CAGMRES_OK;
    }
};

}  // namespace

Transport* make_nccl_transport(const void* unique_id, int rank, int nranks) {
    NcclTransport* t = new (std::nothrow) NcclTransport();
    if (!t) return nullptr;
    ncclUniqueId id;
    std::memcpy(&id, unique_id, sizeof(id));
    if (ncclCommInitRank(&t->comm, nranks, id, rank) != ncclSuccess) {
        t->comm = nullptr;
        delete t;
        return nullptr;
    }
    return t;
}

// ---------------------------------------------------------------------------------------
// In-process group: P rank threads, peer memory.  Every collective is two barrier phases:
//   1. each rank posts its buffers and records `ready` on its stream; barrier;
//      each rank waits on the peers' `ready` events and reads the peers' buffers
//      (peer-to-peer copy or the fixed-order sum kernel), records `done`; barrier;
//   2. each rank waits on the peers' `done` events, so no rank reuses (overwrites) a buffer
//      a peer may still be reading.
// The barrier gives up after a timeout (a rank that failed before a collective would
// otherwise hang the others) and then fails every later collective of the group.
// ---------------------------------------------------------------------------------------
void cagmres_group::barrier() {
    std::unique_lock<std::mutex> lk(mu);
    const uint64_t g0 = gen;
    if (++arrived == P) {
        arrived = 0;
        ++gen;
        cv.notify_all();
        return;
    }
    cv.wait_for(lk, std::chrono::seconds(600), [&] { return gen != g0 || aborted; });
    if (gen == g0) aborted = true;
    cv.notify_all();
}

namespace {

struct GroupTransport final : Transport {
    cagmres_group* g = nullptr;
    int r = 0;
    ~GroupTransport() override {
        // destroy is collective: after the last collective's second barrier a peer may still be
        // enqueueing its waits on our `done` event — no rank destroys its events before every
        // rank has returned from that collective and reached its own destroy
        if (!g->aborted) g->barrier();
        cagmres_group::Post& me = g->post[size_t(r)];
        if (me.ready) cudaEventDestroy(me.ready);
        if (me.done) cudaEventDestroy(me.done);
        cudaFree(me.tmp);
        me = cagmres_group::Post();
        std::lock_guard<std::mutex> lk(g->mu);
        --g->handles;
    }
    int sync_point() {
        g->barrier();
        return g->aborted ? CAGMRES_ENCCL : CAGMRES_OK;
    }
    // phase 2: no peer still reads our buffers once its `done` has completed
    int finish(cudaStream_t st) {
        cagmres_group::Post& me = g->post[size_t(r)];
        if (cudaEventRecord(me.done, st) != cudaSuccess) return CAGMRES_ECUDA;
        if (int e = sync_point()) return e;
        for (int q = 0; q < g->P; ++q)
            if (q != r && cudaStreamWaitEvent(st, g->post[size_t(q)].done, 0) != cudaSuccess) return CAGMRES_ECUDA;
        return CAGMRES_OK;
    }
    int peer_acquire(const void* mine, std::vector<const void*>& all, cudaStream_t st) override {
        cagmres_group::Post& me = g->post[size_t(r)];
        me.ptr = mine;
        me.bytes = 0;
        if (cudaEventRecord(me.ready, st) != cudaSuccess) return CAGMRES_ECUDA;
        if (int e = sync_point()) return e;
        all.assign(size_t(g->P), nullptr);
        for (int q = 0; q < g->P; ++q) {
            if (q != r && cudaStreamWaitEvent(st, g->post[size_t(q)].ready, 0) != cudaSuccess) return CAGMRES_ECUDA;
            all[size_t(q)] = g->post[size_t(q)].ptr;
        }
        return CAGMRES_OK;
    }
    int peer_release(cudaStream_t st) override { return finish(st); }
    bool peer_capable() const override { return true; }
    int allreduce_sum(double* buf, size_t cnt, cudaStream_t st) override {
        cagmres_group::Post& me = g->post[size_t(r)];
        if (cnt > me.tmp_cap) {
            cudaFree(me.tmp);
            me.tmp = nullptr;
            me.tmp_cap = 0;
            if (cudaMalloc(&me.tmp, sizeof(double) * cnt) != cudaSuccess) return CAGMRES_ENOMEM;
            me.tmp_cap = cnt;
        }
        me.ptr = buf;
        me.bytes = sizeof(double) * cnt;
        if (cudaEventRecord(me.ready, st) != cudaSuccess) return CAGMRES_ECUDA;
        if (int e = sync_point()) return e;
        const double* src[16];
        for (int q = 0; q < g->P; ++q) {
            const cagmres_group::Post& o = g->post[size_t(q)];
            if (o.bytes != me.bytes) return CAGMRES_EINVAL;            // ranks disagree on the size
            if (q != r && cudaStreamWaitEvent(st, o.ready, 0) != cudaSuccess) return CAGMRES_ECUDA;
            src[q] = static_cast<const double*>(o.ptr);
        }
        if (cnt) kern::sum_ranks(src, g->P, cnt, me.tmp, st);
        if (int e = finish(st)) return e;
        if (cnt && cudaMemcpyAsync(buf, me.tmp, sizeof(double) * cnt, cudaMemcpyDeviceToDevice, st) != cudaSuccess)
            return CAGMRES_ECUDA;
        return CAGMRES_OK;
    }
    int allgather(const void* send, void* recv, size_t bytes, cudaStream_t st) override {
        cagmres_group::Post& me = g->post[size_t(r)];
        me.ptr = send;
        me.bytes = bytes;
        if (cudaEventRecord(me.ready, st) != cudaSuccess) return CAGMRES_ECUDA;
        if (int e = sync_point()) return e;
        for (int q = 0; q < g->P; ++q) {
            const cagmres_group::Post& o = g->post[size_t(q)];
            if (o.bytes != bytes) return CAGMRES_EINVAL;
            if (q != r && cudaStreamWaitEvent(st, o.ready, 0) != cudaSuccess) return CAGMRES_ECUDA;
            if (bytes && cudaMemcpyAsync(static_cast<char*>(recv) + size_t(q) * bytes, o.ptr, bytes, cudaMemcpyDefault,
                                         st) != cudaSuccess)
                return CAGMRES_ECUDA;
        }
        return finish(st);
    }
    int exchange(const std::vector<Msg>& sends, const std::vector<Msg>& recvs, cudaStream_t st) override {
        cagmres_group::Post& me = g->post[size_t(r)];
        me.sends = sends;
        if (cudaEventRecord(me.ready, st) != cudaSuccess) return CAGMRES_ECUDA;
        if (int e = sync_point()) return e;
        std::vector<int> taken(size_t(g->P), 0), waited(size_t(g->P), 0);
        for (const Msg& m : recvs) {
            if (m.peer < 0 || m.peer >= g->P || m.peer == r) return CAGMRES_EINVAL;
            const std::vector<Msg>& ps = g->post[size_t(m.peer)].sends;
            int seen = 0;
            const Msg* src = nullptr;
            for (const Msg& s : ps)
                if (s.peer == r && seen++ == taken[size_t(m.peer)]) { src = &s; break; }
            if (!src || src->bytes != m.bytes) return CAGMRES_EINVAL;   // unmatched message
            ++taken[size_t(m.peer)];
            if (!waited[size_t(m.peer)]) {
                if (cudaStreamWaitEvent(st, g->post[size_t(m.peer)].ready, 0) != cudaSuccess) return CAGMRES_ECUDA;
                waited[size_t(m.peer)] = 1;
            }
            if (m.bytes && cudaMemcpyAsync(m.ptr, src->ptr, m.bytes, cudaMemcpyDefault, st) != cudaSuccess)
                return CAGMRES_ECUDA;
        }
        return finish(st);
    }
};

}  // namespace

Transport* make_group_transport(cagmres_group* g, int rank) {
    GroupTransport* t = new (std::nothrow) GroupTransport();
    if (!t) return nullptr;
    t->g = g;
    t->r = rank;
    cagmres_group::Post& me = g->post[size_t(rank)];
    if (cudaEventCreateWithFlags(&me.ready, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&me.done, cudaEventDisableTiming) != cudaSuccess) {
        me.ready = me.done = nullptr;
        return nullptr;
    }
    // the sum kernel reads the peers' buffers directly: peer access across devices
    int cur = 0;
    cudaGetDevice(&cur);
    for (int q = 0; q < g->P; ++q) {
        const int d = g->device[size_t(q)];
        if (d == cur) continue;
        int ok = 0;
        cudaDeviceCanAccessPeer(&ok, cur, d);
        if (!ok) return nullptr;
        const cudaError_t e = cudaDeviceEnablePeerAccess(d, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) return nullptr;
        cudaGetLastError();
    }
    {
        std::lock_guard<std::mutex> lk(g->mu);
        ++g->handles;
    }
    return t;
}

namespace kern {

struct SumSrc { const double* p[16]; };

__global__ void k_sum_ranks(SumSrc s, int P, size_t cnt, double* __restrict__ out) {
    for (size_t i = size_t(blockIdx.x) * blockDim.x + threadIdx.x; i < cnt; i += size_t(gridDim.x) * blockDim.x) {
        double a = s.p[0][i];
        for (int q = 1; q < P; ++q) a += s.p[q][i];
        out[i] = a;
    }
}

__global__ void k_sum_chol(SumSrc s, int P, int w, double* __restrict__ G, double* __restrict__ R, int* status) {
    __shared__ double sm[32 * 32];
    pdl_wait();
    pdl_trigger();
    for (int i = threadIdx.x; i < w * w; i += blockDim.x) {
        double a = s.p[0][i];
        for (int q = 1; q < P; ++q) a += s.p[q][i];
        G[i] = a;
    }
    __syncwarp();
    __threadfence_block();
    chol_upper_warp(G, w, w, R, status, sm);
}

void sum_chol(const double* const* src, int P, int w, double* G, double* R, int* status, cudaStream_t st) {
    SumSrc s{};
    for (int q = 0; q < P && q < 16; ++q) s.p[q] = src[q];
    ++g_launches;
    launch_pdl(k_sum_chol, dim3(1), dim3(32), 0, st, s, P, w, G, R, status);
}

__global__ void k_halo_pull(PullSegs sg, int64_t tot, const int64_t* __restrict__ loc,
                            const int64_t* __restrict__ ext, double* __restrict__ dst) {
    for (int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; t < tot; t += int64_t(gridDim.x) * blockDim.x) {
        int i = 0;
        int64_t k = t;
        while (k >= sg.cnt[i]) { k -= sg.cnt[i]; ++i; }
        k += sg.off[i];
        dst[ext[k]] = sg.src[i][loc[k]];
    }
}

void halo_pull(const PullSegs& sg, const int64_t* loc, const int64_t* ext, double* dst, cudaStream_t st) {
    int64_t tot = 0;
    for (int i = 0; i < sg.n; ++i) tot += sg.cnt[i];
    if (tot <= 0) return;
    const int64_t g = std::min<int64_t>((tot + 255) / 256, 4096);
    ++g_launches;
    k_halo_pull<<<unsigned(g), 256, 0, st>>>(sg, tot, loc, ext, dst);
}

void sum_ranks(const double* const* src, int P, size_t cnt, double* out, cudaStream_t st) {
    SumSrc s{};
    for (int q = 0; q < P && q < 16; ++q) s.p[q] = src[q];
    const size_t g = std::min<size_t>((cnt + 255) / 256, 1024);
    ++g_launches;
    k_sum_ranks<<<unsigned(g), 256, 0, st>>>(s, P, cnt, out);
}

}  // namespace kern

// ---------------------------------------------------------------------------------------
// C ABI
// ---------------------------------------------------------------------------------------
extern "C" {

int cagmres_group_create(cagmres_group_t* out, int nranks, const int* devices) {
    if (!out || nranks < 1 || nranks > 16) return CAGMRES_EINVAL;
    *out = nullptr;
    cagmres_group* g = new (std::nothrow) cagmres_group();
    if (!g) return CAGMRES_ENOMEM;
    g->P = nranks;
    g->device.assign(size_t(nranks), 0);
    if (devices) {
        int nd = 0;
        if (cudaGetDeviceCount(&nd) != cudaSuccess) nd = 0;
        for (int q = 0; q < nranks; ++q) {
            if (devices[q] < 0 || (nd > 0 && devices[q] >= nd)) { delete g; return CAGMRES_EINVAL; }
            g->device[size_t(q)] = devices[q];
        }
    }
    g->post.resize(size_t(nranks));
    *out = g;
    return CAGMRES_OK;
}

int cagmres_group_destroy(cagmres_group_t g) {
    if (!g) return CAGMRES_OK;
    {
        std::lock_guard<std::mutex> lk(g->mu);
        if (g->handles > 0) return CAGMRES_EINVAL;      // a handle still uses the group
    }
    delete g;
    return CAGMRES_OK;
}

}  // extern "C"
