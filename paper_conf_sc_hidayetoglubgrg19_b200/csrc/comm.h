// comm.h -- the multi-GPU transport of the domain decomposition A = R C A_p.
//
// Two implementations of one interface:
//   * NcclComm  -- one process per GPU; NCCL (dlopen'ed libnccl.so.2) grouped ncclSend/ncclRecv
//                  as the sparse all-to-allv of P:731-756, ncclAllReduce for CG dot products.
//                  All calls are stream-ordered and CUDA-graph capturable.
//   * LocalComm -- P "virtual ranks" (plans) in one process on one device, one host thread
//                  each; the same collectives done with device-to-device copies and a small
//                  device reduction kernel.  A test shim: it lets the whole multi-rank path run
//                  and be checked against the oracle on a single GPU.  Not graph-capturable.
#pragma once

#include <condition_variable>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "common.h"

namespace mx {

enum class DType { I32, I64, F32, F64 };
size_t dtype_size(DType t);

class Comm {
public:
    virtual ~Comm() = default;
    int rank = 0, nranks = 1;
    virtual bool capturable() const = 0;
    // in-place elementwise sum over ranks (device buffer)
    virtual void allreduce_sum(void* buf, int64_t count, DType t, cudaStream_t st) = 0;
    // sparse all-to-allv: to peer q send `scount[q]` elements at send + sdispl[q], from peer q
    // receive `rcount[q]` elements into recv + rdispl[q] (host count/displacement arrays).
    virtual void alltoallv(const void* send, const int64_t* scount, const int64_t* sdispl, void* recv,
                           const int64_t* rcount, const int64_t* rdispl, DType t, cudaStream_t st) = 0;
    // dense collectives (EXCHANGE = 2, the comparison of SURVEY 8(e)): every rank's `send` holds
    // nranks blocks of `count` elements; rank g receives the elementwise sum over ranks of block g
    virtual void reduce_scatter_sum(const void* send, void* recv, int64_t count, DType t, cudaStream_t st) = 0;
    // every rank contributes `count` elements; recv = the nranks contributions in rank order
    virtual void allgather(const void* send, void* recv, int64_t count, DType t, cudaStream_t st) = 0;
    // gather one int64 per rank on the host (build-time bookkeeping)
    virtual std::vector<int64_t> allgather_host(int64_t v, cudaStream_t st) = 0;
    // gather a vector of n int64 per rank: out[q * n + i] (build-time)
    virtual std::vector<int64_t> allgather_vec(const std::vector<int64_t>& v, cudaStream_t st) = 0;
    // Peer memory: every rank passes a cudaMalloc'ed device buffer; returns each rank's buffer as
    // a pointer this rank's kernels can load/store (NVLink peer mapping via CUDA IPC for NCCL
    // ranks, the plain pointer for virtual ranks).  Collective.  Throws if peers are unreachable.
    virtual std::vector<void*> map_peers(void* local, cudaStream_t st) = 0;
    // Host poll of asynchronous transport errors (NCCL: ncclCommGetAsyncError); throws
    // MEMXCT_ERR_NCCL.  Called at the start of every library call on a decomposed plan.
    virtual void check_async() {}
    // true when every rank runs on this rank's device (virtual ranks, or host-transport processes
    // sharing a GPU): the fused exchange then keeps its waits in one-thread kernels
    virtual bool shares_device() const { return false; }
};

std::unique_ptr<Comm> make_nccl_comm(int rank, int nranks, const void* unique_id);
// processes of one node (possibly sharing a GPU) over a named POSIX shared-memory segment and
// CUDA IPC device mailboxes (proccomm.cu); not graph-capturable
std::unique_ptr<Comm> make_host_comm(const std::string& name, int rank, int nranks);
// host-only round trip of the host transport (rendezvous, barriers, host allgather): no device
std::vector<int64_t> host_comm_probe(const std::string& name, int rank, int nranks, int64_t value);
void nccl_unique_id(void* out);

// shared state of a group of virtual ranks
struct LocalGroup {
    explicit LocalGroup(int n) : nranks(n), posts(n) {}
    int nranks;
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    int64_t generation = 0;
    struct Post {
        const void* send = nullptr;
        const int64_t* sdispl = nullptr;
        const int64_t* scount = nullptr;
        void* buf = nullptr;
        int64_t value = 0;
        const std::vector<int64_t>* vec = nullptr;
    };
    std::vector<Post> posts;
    void barrier();
};

std::unique_ptr<Comm> make_local_comm(std::shared_ptr<LocalGroup> g, int rank);

}  // namespace mx
