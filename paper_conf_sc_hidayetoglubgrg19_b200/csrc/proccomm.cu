// proccomm.cu -- the host transport of the decomposition across PROCESSES of one node
// (memxct_plan_set_comm_host): one process per rank, ranks may share a GPU.
//
// The multi-GPU data plane of A = R C A_p is NCCL's in production (comm.cu), but NCCL
// refuses two ranks on one device, and the sandbox this library is developed in offers one GPU.
// This transport lets two or more processes on ONE device run the real cross-process path: the
// fused peer exchange (EXCHANGE = 1) maps the other processes' buffers with cudaIpcOpenMemHandle
// and synchronises through system-scope flags and credits exactly as NCCL ranks do, and the
// collective exchanges move data between processes through IPC-mapped device mailboxes.
//
//   rendezvous  a POSIX shared-memory segment named by the caller (rank 0 creates and
//               initialises it; the others attach once it is marked ready; rank 0 unlinks the
//               name as soon as every rank is attached);
//   barrier     sense-counting spin barrier on process-shared atomics, with a time-out
//               (MEMXCT_ERR_NCCL instead of hanging when a peer process is gone);
//   host data   per-rank slots in the segment (allgather of int64 vectors);
//   device data every rank's device mailbox, exported once by CUDA IPC and opened by the others;
//               a collective copies its input into the own mailbox, barriers, and pulls what it
//               needs from the peers' mailboxes (device-to-device copies), then barriers again
//               before anyone reuses a mailbox.  Sums over ranks run in rank order (the same
//               fixed-order kernel as the virtual ranks, so results are bit-identical to them).
// Not graph-capturable (host barriers inside the collectives), like the virtual ranks.
#include <fcntl.h>
#include <sched.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <atomic>
#include <chrono>
#include <cstring>
#include <string>
#include <thread>

#include "comm.h"

namespace mx {

namespace {

constexpr int kMaxRanks = 16;                    // kMaxPeers of the fused exchange
constexpr int64_t kSlotWords = 1 << 14;          // host allgather slot: 128 KB per rank (~2 MB segment)
constexpr uint64_t kMagic = 0x4d454d5843543031ull;  // "MEMXCT01"
// rendezvous / barrier time-out: 300 s, or MEMXCT_HOST_COMM_TIMEOUT_S (tests)
double timeout_s() {
    static const double v = [] {
        const char* e = std::getenv("MEMXCT_HOST_COMM_TIMEOUT_S");
        return e ? std::max(0.1, atof(e)) : 300.0;
    }();
    return v;
}

struct Shared {
    std::atomic<uint64_t> magic;
    int32_t nranks;
    std::atomic<int64_t> arrived;
    std::atomic<int64_t> generation;
    // per rank: the current device mailbox (IPC handle + size + version), a scalar, a vector
    struct Rank {
        cudaIpcMemHandle_t mbox;
        int64_t mbox_bytes;
        int64_t mbox_version;
        int64_t need;
        int64_t scount[kMaxRanks], sdispl[kMaxRanks];
        int64_t nwords;
        char device_uuid[16];
    } rank[kMaxRanks];
    int64_t words[kMaxRanks][kSlotWords];
};

template <class T>
__global__ void sum_ranks_proc_kernel(const T* __restrict__ tmp, int nr, int64_t count, T* __restrict__ out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        T s = tmp[i];
        for (int q = 1; q < nr; ++q) s += tmp[(int64_t)q * count + i];  // fixed rank order
        out[i] = s;
    }
}

class ProcComm : public Comm {
public:
    ProcComm(const std::string& name, int r, int n) : name_(name) {
        rank = r;
        nranks = n;
        if (n < 1 || n > kMaxRanks) fail(MEMXCT_ERR_INVALID_ARG, "host transport: 1..16 ranks");
        const size_t bytes = sizeof(Shared);
        const auto t0 = std::chrono::steady_clock::now();
        int fd = -1;
        if (r == 0) {
            fd = shm_open(name.c_str(), O_CREAT | O_EXCL | O_RDWR, 0600);
            if (fd < 0) fail(MEMXCT_ERR_INVALID_ARG, "host transport: shm_open(" + name + ") failed (name in use?)");
            if (ftruncate(fd, (off_t)bytes) != 0) {
                close(fd);
                fail(MEMXCT_ERR_OUT_OF_MEMORY, "host transport: ftruncate failed");
            }
        } else {
            while ((fd = shm_open(name.c_str(), O_RDWR, 0600)) < 0) {
                if (elapsed(t0) > timeout_s()) fail(MEMXCT_ERR_NCCL, "host transport: rank 0 never created " + name);
                std::this_thread::sleep_for(std::chrono::milliseconds(2));
            }
            struct stat sb;
            while (fstat(fd, &sb) == 0 && (size_t)sb.st_size < bytes) {
                if (elapsed(t0) > timeout_s()) fail(MEMXCT_ERR_NCCL, "host transport: segment never sized");
                std::this_thread::sleep_for(std::chrono::milliseconds(2));
            }
        }
        void* p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
        close(fd);
        if (p == MAP_FAILED) fail(MEMXCT_ERR_OUT_OF_MEMORY, "host transport: mmap failed");
        sh_ = static_cast<Shared*>(p);
        if (r == 0) {
            sh_->nranks = n;
            sh_->arrived.store(0);
            sh_->generation.store(0);
            sh_->magic.store(kMagic, std::memory_order_release);
        } else {
            while (sh_->magic.load(std::memory_order_acquire) != kMagic) {
                if (elapsed(t0) > timeout_s()) fail(MEMXCT_ERR_NCCL, "host transport: segment never initialised");
                std::this_thread::sleep_for(std::chrono::milliseconds(2));
            }
            if (sh_->nranks != n) fail(MEMXCT_ERR_INVALID_ARG, "host transport: nranks differs from rank 0's");
        }
        // the device's UUID (zeros without a device: the host-only probe, memxct_host_comm_probe)
        std::memset(sh_->rank[rank].device_uuid, 0, 16);
        int dev = 0;
        cudaDeviceProp prop;
        if (cudaGetDevice(&dev) == cudaSuccess && cudaGetDeviceProperties(&prop, dev) == cudaSuccess)
            std::memcpy(sh_->rank[rank].device_uuid, &prop.uuid, 16);
        else
            cudaGetLastError();
        barrier();
        if (r == 0) shm_unlink(name.c_str());  // every rank is attached: the name is no longer needed
        same_device_ = true;
        for (int q = 0; q < nranks; ++q)
            same_device_ = same_device_ && !std::memcmp(sh_->rank[q].device_uuid, sh_->rank[rank].device_uuid, 16);
    }
    ~ProcComm() override {
        for (void* q : opened_) cudaIpcCloseMemHandle(q);
        if (sh_) munmap(sh_, sizeof(Shared));
    }
    bool capturable() const override { return false; }
    bool shares_device() const override { return same_device_; }

    void allreduce_sum(void* buf, int64_t count, DType t, cudaStream_t st) override {
        const size_t es = dtype_size(t), b = es * (size_t)count;
        post_mailbox(buf, b, st);
        grow_scratch(b * nranks);
        for (int q = 0; q < nranks; ++q)
            if (b) MX_CUDA(cudaMemcpyAsync(scratch_.as<char>() + q * b, peer_mbox(q), b, cudaMemcpyDeviceToDevice, st));
        MX_CUDA(cudaStreamSynchronize(st));
        barrier();  // every rank has read every mailbox
        sum_into(scratch_.get(), buf, count, t, st);
    }

    void reduce_scatter_sum(const void* send, void* recv, int64_t count, DType t, cudaStream_t st) override {
        const size_t es = dtype_size(t), b = es * (size_t)count;
        post_mailbox(send, b * nranks, st);
        grow_scratch(b * nranks);
        for (int q = 0; q < nranks; ++q)
            if (b) MX_CUDA(cudaMemcpyAsync(scratch_.as<char>() + q * b, peer_mbox(q) + rank * b, b,
                                           cudaMemcpyDeviceToDevice, st));
        MX_CUDA(cudaStreamSynchronize(st));
        barrier();
        sum_into(scratch_.get(), recv, count, t, st);
    }

    void allgather(const void* send, void* recv, int64_t count, DType t, cudaStream_t st) override {
        const size_t b = dtype_size(t) * (size_t)count;
        post_mailbox(send, b, st);
        for (int q = 0; q < nranks; ++q)
            if (b) MX_CUDA(cudaMemcpyAsync(static_cast<char*>(recv) + q * b, peer_mbox(q), b, cudaMemcpyDeviceToDevice, st));
        MX_CUDA(cudaStreamSynchronize(st));
        barrier();
    }

    void alltoallv(const void* send, const int64_t* scount, const int64_t* sdispl, void* recv,
                   const int64_t* rcount, const int64_t* rdispl, DType t, cudaStream_t st) override {
        const size_t es = dtype_size(t);
        int64_t extent = 0;
        for (int q = 0; q < nranks; ++q) {
            extent = std::max(extent, sdispl[q] + scount[q]);
            sh_->rank[rank].scount[q] = scount[q];
            sh_->rank[rank].sdispl[q] = sdispl[q];
        }
        post_mailbox(send, es * (size_t)extent, st);
        for (int q = 0; q < nranks; ++q) {
            if (sh_->rank[q].scount[rank] != rcount[q]) fail(MEMXCT_ERR_CUDA, "internal: all-to-allv count mismatch");
            if (rcount[q] > 0)
                MX_CUDA(cudaMemcpyAsync(static_cast<char*>(recv) + rdispl[q] * es,
                                        peer_mbox(q) + sh_->rank[q].sdispl[rank] * es, rcount[q] * es,
                                        cudaMemcpyDeviceToDevice, st));
        }
        MX_CUDA(cudaStreamSynchronize(st));
        barrier();
    }

    std::vector<int64_t> allgather_host(int64_t v, cudaStream_t st) override {
        return allgather_vec(std::vector<int64_t>{v}, st);
    }

    std::vector<int64_t> allgather_vec(const std::vector<int64_t>& v, cudaStream_t) override {
        if ((int64_t)v.size() > kSlotWords) fail(MEMXCT_ERR_UNSUPPORTED, "host transport: vector beyond 128 KB");
        sh_->rank[rank].nwords = (int64_t)v.size();
        std::memcpy(sh_->words[rank], v.data(), 8 * v.size());
        barrier();
        std::vector<int64_t> out;
        for (int q = 0; q < nranks; ++q)
            out.insert(out.end(), sh_->words[q], sh_->words[q] + sh_->rank[q].nwords);
        barrier();
        return out;
    }

    std::vector<void*> map_peers(void* local, cudaStream_t st) override {
        cudaIpcMemHandle_t h;
        MX_CUDA(cudaIpcGetMemHandle(&h, local));
        std::vector<int64_t> words(sizeof(h) / 8);
        std::memcpy(words.data(), &h, sizeof(h));
        const auto all = allgather_vec(words, st);
        std::vector<void*> out(nranks, nullptr);
        std::string err;
        for (int q = 0; q < nranks && err.empty(); ++q) {
            if (q == rank) { out[q] = local; continue; }
            cudaIpcMemHandle_t hq;
            std::memcpy(&hq, all.data() + q * words.size(), sizeof(hq));
            void* p = nullptr;
            const cudaError_t e = cudaIpcOpenMemHandle(&p, hq, cudaIpcMemLazyEnablePeerAccess);
            if (e != cudaSuccess) {
                cudaGetLastError();
                err = std::string("cudaIpcOpenMemHandle(peer ") + std::to_string(q) + "): " + cudaGetErrorString(e);
                break;
            }
            opened_.push_back(p);
            out[q] = p;
        }
        const auto ok = allgather_host(err.empty() ? 1 : 0, st);
        for (int64_t v : ok)
            if (!v) fail(MEMXCT_ERR_UNSUPPORTED, err.empty() ? "peer mapping failed on another rank" : err);
        return out;
    }

    void barrier() {
        const int64_t gen = sh_->generation.load(std::memory_order_acquire);
        if (sh_->arrived.fetch_add(1, std::memory_order_acq_rel) + 1 == nranks) {
            sh_->arrived.store(0, std::memory_order_relaxed);
            sh_->generation.fetch_add(1, std::memory_order_acq_rel);
            return;
        }
        const auto t0 = std::chrono::steady_clock::now();
        int spins = 0;
        while (sh_->generation.load(std::memory_order_acquire) == gen) {
            if (++spins > 1000) std::this_thread::sleep_for(std::chrono::microseconds(20));
            else sched_yield();
            if (spins % 4096 == 0 && elapsed(t0) > timeout_s())
                fail(MEMXCT_ERR_NCCL, "host transport: a peer process did not reach the barrier");
        }
    }

private:
    static double elapsed(std::chrono::steady_clock::time_point t0) {
        return std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    }

    // copy `bytes` of `src` into this rank's mailbox (grown collectively if any rank needs more),
    // then barrier: afterwards every rank may read every mailbox
    void post_mailbox(const void* src, size_t bytes, cudaStream_t st) {
        MX_CUDA(cudaStreamSynchronize(st));
        sh_->rank[rank].need = (int64_t)bytes;
        barrier();
        int64_t need = 0;
        for (int q = 0; q < nranks; ++q) need = std::max(need, sh_->rank[q].need);
        if (need > mbox_bytes_) {
            // grow-only: the previous mailbox stays allocated (no cudaFree, which would wait for
            // the whole device) and the peers' previous mappings stay open until destruction
            if (mbox_.get()) retired_.push_back(std::move(mbox_));
            mbox_.alloc((size_t)std::max<int64_t>(need, (int64_t)64 << 20));
            mbox_bytes_ = (int64_t)mbox_.bytes();
            MX_CUDA(cudaIpcGetMemHandle(&sh_->rank[rank].mbox, mbox_.get()));
            sh_->rank[rank].mbox_bytes = mbox_bytes_;
            sh_->rank[rank].mbox_version = ++version_;
            barrier();
            peers_.assign(nranks, nullptr);
            for (int q = 0; q < nranks; ++q) {
                if (q == rank) { peers_[q] = mbox_.get(); continue; }
                void* p = nullptr;
                MX_CUDA(cudaIpcOpenMemHandle(&p, sh_->rank[q].mbox, cudaIpcMemLazyEnablePeerAccess));
                opened_.push_back(p);
                peers_[q] = p;
            }
        }
        if (bytes) MX_CUDA(cudaMemcpyAsync(mbox_.get(), src, bytes, cudaMemcpyDeviceToDevice, st));
        MX_CUDA(cudaStreamSynchronize(st));
        barrier();
    }
    const char* peer_mbox(int q) const { return static_cast<const char*>(peers_[q]); }
    void grow_scratch(size_t b) {
        if (scratch_.bytes() < std::max(b, (size_t)4096)) {
            if (scratch_.get()) retired_.push_back(std::move(scratch_));
            scratch_.alloc(std::max(b, (size_t)4096));
        }
    }
    void sum_into(const void* tmp, void* out, int64_t count, DType t, cudaStream_t st) {
        if (count > 0) {
            const unsigned blocks = (unsigned)std::min<int64_t>(1024, ceil_div(count, 256));
            switch (t) {
                case DType::I32: sum_ranks_proc_kernel<<<blocks, 256, 0, st>>>((const int32_t*)tmp, nranks, count, (int32_t*)out); break;
                case DType::I64: sum_ranks_proc_kernel<<<blocks, 256, 0, st>>>((const int64_t*)tmp, nranks, count, (int64_t*)out); break;
                case DType::F32: sum_ranks_proc_kernel<<<blocks, 256, 0, st>>>((const float*)tmp, nranks, count, (float*)out); break;
                case DType::F64: sum_ranks_proc_kernel<<<blocks, 256, 0, st>>>((const double*)tmp, nranks, count, (double*)out); break;
            }
            MX_LAUNCHED();
        }
        MX_CUDA(cudaStreamSynchronize(st));
    }

    std::string name_;
    Shared* sh_ = nullptr;
    bool same_device_ = false;
    DevBuf mbox_, scratch_;
    int64_t mbox_bytes_ = 0, version_ = 0;
    std::vector<void*> peers_, opened_;
    std::vector<DevBuf> retired_;
};

}  // namespace

std::unique_ptr<Comm> make_host_comm(const std::string& name, int rank, int nranks) {
    return std::make_unique<ProcComm>(name, rank, nranks);
}

std::vector<int64_t> host_comm_probe(const std::string& name, int rank, int nranks, int64_t value) {
    ProcComm c(name, rank, nranks);
    auto v = c.allgather_host(value, nullptr);
    c.barrier();
    return v;
}


}  // namespace mx
