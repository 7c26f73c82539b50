// transport.h — the communication seam under the distributed handle (not part of the C ABI).
//
// The distributed CA-GMRES cycle needs three kinds of exchange:
//   * the MPK halo: grouped point-to-point messages to the owners / requesters of ghost rows
//     (Fig. 4 setup), and the request-list exchange of the setup;
//   * sums of the BOrth coefficients and the w x w Gram over all ranks;
//   * an all-gather of per-rank counts (setup).
// Two implementations:
//   * Nccl   — one process per GPU, NCCL over NVLink/NVSwitch (the production multi-GPU path);
//   * Group  — P ranks inside ONE process (one host thread per rank), each rank on its own
//              device or all on the same device: messages are peer-to-peer cudaMemcpyAsync
//              (NVLink when the devices differ), sums are one fixed-order kernel per rank that
//              reads every rank's buffer directly.  With one GPU this runs the complete
//              multi-rank device path (pack -> exchange -> unpack, allreduce -> Cholesky, the
//              distributed residual) on a single device.
// All calls are stream-ordered on the caller's stream and must be made by every rank in the
// same order (the same contract as NCCL).
#pragma once
#include <condition_variable>
#include <cstddef>
#include <cstdint>
#include <mutex>
#include <vector>

#include <cuda_runtime.h>

struct Msg {
    int peer;
    void* ptr;          // device
    size_t bytes;
};

struct Transport {
    virtual ~Transport() = default;
    // buf[0:cnt) := sum over ranks (identical bits on every rank)
    virtual int allreduce_sum(double* buf, size_t cnt, cudaStream_t st) = 0;
    // recv[q * bytes : (q+1) * bytes) := rank q's send[0:bytes)   (device buffers)
    virtual int allgather(const void* send, void* recv, size_t bytes, cudaStream_t st) = 0;
    // grouped send / recv; the k-th send to a peer matches that peer's k-th recv from us
    virtual int exchange(const std::vector<Msg>& sends, const std::vector<Msg>& recvs, cudaStream_t st) = 0;
    // One-sided peer access (in-process group only; NCCL: ENOTSUP).  peer_acquire posts `mine`,
    // makes the stream wait until every rank's buffer is complete and returns all ranks'
    // pointers (device-loadable: same device or peer access enabled); the caller then launches
    // ONE kernel that reads the peers' buffers directly (the halo pull, the fused cross-rank
    // sum + Cholesky) and calls peer_release, after which no rank reuses its buffer before
    // every reader is done.  Same calling contract as the collectives.
    virtual int peer_acquire(const void* mine, std::vector<const void*>& all, cudaStream_t st) {
        (void)mine; (void)all; (void)st;
        return -7;   // CAGMRES_ENOTSUP
    }
    virtual int peer_release(cudaStream_t st) { (void)st; return -7; }
    virtual bool peer_capable() const { return false; }
};

// NCCL communicator from a 128-byte ncclUniqueId; nullptr on failure.
Transport* make_nccl_transport(const void* unique_id, int rank, int nranks);

// In-process group shared by P rank threads (C ABI: cagmres_group_t).
struct cagmres_group {
    int P = 1;
    std::vector<int> device;                  // device of each rank
    // generation barrier
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    uint64_t gen = 0;
    bool aborted = false;                     // a barrier timed out: every later collective fails
    // what every rank posted for the current collective
    struct Post {
        const void* ptr = nullptr;
        size_t bytes = 0;
        std::vector<Msg> sends;
        cudaEvent_t ready = nullptr, done = nullptr;
        double* tmp = nullptr;                 // allreduce result scratch (on the rank's device)
        size_t tmp_cap = 0;
    };
    std::vector<Post> post;
    int handles = 0;                          // live transports created from this group
    void barrier();
};

Transport* make_group_transport(cagmres_group* g, int rank);

namespace kern {
// out[0:cnt) = src[0][.] + src[1][.] + ... + src[P-1][.] in this order (P <= 16)
void sum_ranks(const double* const* src, int P, size_t cnt, double* out, cudaStream_t st);
// G = sum over ranks of the w x w Grams src[q] (rank order), R = chol(G) (upper, ld w) in ONE
// launch (one warp); breakdown sets ST_CHOL in *status
void sum_chol(const double* const* src, int P, int w, double* G, double* R, int* status, cudaStream_t st);
// Halo pull over peer memory: for each segment i (one per owner rank) and k in
// [off[i], off[i] + cnt[i]): dst[ext[k]] = src_i[loc[k]] — owner-local index loc, extended
// row ext.  One launch replaces pack -> P-1 copies -> unpack.
struct PullSegs {
    const double* src[16];
    int64_t off[16], cnt[16];
    int n = 0;
};
void halo_pull(const PullSegs& sg, const int64_t* loc, const int64_t* ext, double* dst, cudaStream_t st);
}
