// comm.cu -- NCCL transport (dlopen'ed) and the in-process virtual-rank shim (see comm.h).
#include <dlfcn.h>
#include <nccl.h>

#include <cstring>
#include <string>

#include "comm.h"

namespace mx {

size_t dtype_size(DType t) {
    switch (t) {
        case DType::I32: case DType::F32: return 4;
        default: return 8;
    }
}

// ------------------------------------------------------------------------------------------
// NCCL
// ------------------------------------------------------------------------------------------
namespace {

struct NcclApi {
    decltype(&ncclGetUniqueId) GetUniqueId = nullptr;
    decltype(&ncclCommInitRank) CommInitRank = nullptr;
    decltype(&ncclCommDestroy) CommDestroy = nullptr;
    decltype(&ncclAllReduce) AllReduce = nullptr;
    decltype(&ncclAllGather) AllGather = nullptr;
    decltype(&ncclReduceScatter) ReduceScatter = nullptr;
    decltype(&ncclSend) Send = nullptr;
    decltype(&ncclRecv) Recv = nullptr;
    decltype(&ncclGroupStart) GroupStart = nullptr;
    decltype(&ncclGroupEnd) GroupEnd = nullptr;
    decltype(&ncclGetErrorString) GetErrorString = nullptr;
    decltype(&ncclCommGetAsyncError) GetAsyncError = nullptr;
    std::string error;

    static NcclApi& get() {
        static NcclApi api = load();
        return api;
    }
    static NcclApi load() {
        NcclApi a;
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            a.error = std::string("dlopen(libnccl.so.2) failed: ") + dlerror();
            return a;
        }
#define MX_SYM(field, name) a.field = reinterpret_cast<decltype(a.field)>(dlsym(h, name))
        MX_SYM(GetUniqueId, "ncclGetUniqueId");
        MX_SYM(CommInitRank, "ncclCommInitRank");
        MX_SYM(CommDestroy, "ncclCommDestroy");
        MX_SYM(AllReduce, "ncclAllReduce");
        MX_SYM(AllGather, "ncclAllGather");
        MX_SYM(ReduceScatter, "ncclReduceScatter");
        MX_SYM(Send, "ncclSend");
        MX_SYM(Recv, "ncclRecv");
        MX_SYM(GroupStart, "ncclGroupStart");
        MX_SYM(GroupEnd, "ncclGroupEnd");
        MX_SYM(GetErrorString, "ncclGetErrorString");
        MX_SYM(GetAsyncError, "ncclCommGetAsyncError");
#undef MX_SYM
        if (!a.GetUniqueId || !a.CommInitRank || !a.AllReduce || !a.Send || !a.Recv || !a.GroupStart ||
            !a.GroupEnd || !a.AllGather || !a.ReduceScatter || !a.CommDestroy)
            a.error = "libnccl.so.2 lacks required symbols";
        return a;
    }
    void check(ncclResult_t r, const char* what) const {
        if (r != ncclSuccess)
            fail(MEMXCT_ERR_NCCL, std::string(what) + ": " + (GetErrorString ? GetErrorString(r) : "error"));
    }
};

NcclApi& nccl() {
    NcclApi& a = NcclApi::get();
    if (!a.error.empty()) fail(MEMXCT_ERR_NCCL, a.error);
    return a;
}

ncclDataType_t nccl_type(DType t) {
    switch (t) {
        case DType::I32: return ncclInt32;
        case DType::I64: return ncclInt64;
        case DType::F32: return ncclFloat32;
        default: return ncclFloat64;
    }
}

class NcclComm : public Comm {
public:
    NcclComm(int r, int n, const void* uid) {
        rank = r;
        nranks = n;
        ncclUniqueId id;
        std::memcpy(&id, uid, sizeof(id));
        nccl().check(nccl().CommInitRank(&comm_, n, id, r), "ncclCommInitRank");
    }
    ~NcclComm() override {
        for (void* p : opened_) cudaIpcCloseMemHandle(p);
        if (comm_) NcclApi::get().CommDestroy(comm_);
    }
    bool capturable() const override { return true; }
    void check_async() override {
        NcclApi& a = nccl();
        if (!a.GetAsyncError || !comm_) return;
        ncclResult_t r = ncclSuccess;
        a.check(a.GetAsyncError(comm_, &r), "ncclCommGetAsyncError");
        if (r != ncclSuccess && r != ncclInProgress) a.check(r, "NCCL asynchronous error");
    }
    void allreduce_sum(void* buf, int64_t count, DType t, cudaStream_t st) override {
        if (count == 0) return;
        nccl().check(nccl().AllReduce(buf, buf, (size_t)count, nccl_type(t), ncclSum, comm_, st), "ncclAllReduce");
    }
    void reduce_scatter_sum(const void* send, void* recv, int64_t count, DType t, cudaStream_t st) override {
        if (count == 0) return;
        nccl().check(nccl().ReduceScatter(send, recv, (size_t)count, nccl_type(t), ncclSum, comm_, st),
                     "ncclReduceScatter");
    }
    void allgather(const void* send, void* recv, int64_t count, DType t, cudaStream_t st) override {
        if (count == 0) return;
        nccl().check(nccl().AllGather(send, recv, (size_t)count, nccl_type(t), comm_, st), "ncclAllGather");
    }
    void alltoallv(const void* send, const int64_t* scount, const int64_t* sdispl, void* recv,
                   const int64_t* rcount, const int64_t* rdispl, DType t, cudaStream_t st) override {
        const size_t es = dtype_size(t);
        if (scount[rank] > 0)
            MX_CUDA(cudaMemcpyAsync(static_cast<char*>(recv) + rdispl[rank] * es,
                                    static_cast<const char*>(send) + sdispl[rank] * es, scount[rank] * es,
                                    cudaMemcpyDeviceToDevice, st));
        NcclApi& a = nccl();
        a.check(a.GroupStart(), "ncclGroupStart");
        for (int q = 0; q < nranks; ++q) {
            if (q == rank) continue;
            if (scount[q] > 0)
                a.check(a.Send(static_cast<const char*>(send) + sdispl[q] * es, (size_t)scount[q], nccl_type(t), q,
                               comm_, st), "ncclSend");
            if (rcount[q] > 0)
                a.check(a.Recv(static_cast<char*>(recv) + rdispl[q] * es, (size_t)rcount[q], nccl_type(t), q,
                               comm_, st), "ncclRecv");
        }
        a.check(a.GroupEnd(), "ncclGroupEnd");
    }
    std::vector<int64_t> allgather_host(int64_t v, cudaStream_t st) override {
        return allgather_vec(std::vector<int64_t>{v}, st);
    }
    std::vector<int64_t> allgather_vec(const std::vector<int64_t>& v, cudaStream_t st) override {
        const int64_t n = (int64_t)v.size();
        DevArr<int64_t> d;
        d.alloc(n * (nranks + 1));
        int64_t* mine = d.p() + n * nranks;
        if (n > 0) MX_CUDA(cudaMemcpyAsync(mine, v.data(), 8 * n, cudaMemcpyHostToDevice, st));
        nccl().check(nccl().AllGather(mine, d.p(), (size_t)n, ncclInt64, comm_, st), "ncclAllGather");
        std::vector<int64_t> h(n * nranks);
        if (n > 0) MX_CUDA(cudaMemcpyAsync(h.data(), d.p(), 8 * n * nranks, cudaMemcpyDeviceToHost, st));
        MX_CUDA(cudaStreamSynchronize(st));
        return h;
    }
    std::vector<void*> map_peers(void* local, cudaStream_t st) override {
        cudaIpcMemHandle_t h;
        MX_CUDA(cudaIpcGetMemHandle(&h, local));
        static_assert(sizeof(h) % 8 == 0, "IPC handle size");
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
        // agree on success before anyone goes on (a one-sided failure would hang the others)
        const auto ok = allgather_host(err.empty() ? 1 : 0, st);
        for (int64_t v : ok)
            if (!v) fail(MEMXCT_ERR_UNSUPPORTED, err.empty() ? "peer mapping failed on another rank" : err);
        return out;
    }

private:
    ncclComm_t comm_ = nullptr;
    std::vector<void*> opened_;
};

}  // namespace

std::unique_ptr<Comm> make_nccl_comm(int rank, int nranks, const void* unique_id) {
    return std::make_unique<NcclComm>(rank, nranks, unique_id);
}

void nccl_unique_id(void* out) {
    ncclUniqueId id;
    nccl().check(nccl().GetUniqueId(&id), "ncclGetUniqueId");
    std::memcpy(out, &id, sizeof(id));
}

// ------------------------------------------------------------------------------------------
// virtual ranks in one process
// ------------------------------------------------------------------------------------------
void LocalGroup::barrier() {
    std::unique_lock<std::mutex> lk(mu);
    const int64_t gen = generation;
    if (++arrived == nranks) {
        arrived = 0;
        ++generation;
        cv.notify_all();
    } else {
        cv.wait(lk, [&] { return generation != gen; });
    }
}

namespace {

template <class T>
__global__ void sum_ranks_kernel(const T* __restrict__ tmp, int nr, int64_t count, T* __restrict__ out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        T s = tmp[i];
        for (int q = 1; q < nr; ++q) s += tmp[(int64_t)q * count + i];  // fixed rank order
        out[i] = s;
    }
}

class LocalComm : public Comm {
public:
    LocalComm(std::shared_ptr<LocalGroup> g, int r) : g_(std::move(g)) {
        rank = r;
        nranks = g_->nranks;
    }
    bool capturable() const override { return false; }
    bool shares_device() const override { return true; }

    void allreduce_sum(void* buf, int64_t count, DType t, cudaStream_t st) override {
        MX_CUDA(cudaStreamSynchronize(st));
        const size_t es = dtype_size(t);
        g_->posts[rank].buf = buf;
        g_->barrier();
        // grow-only scratch: a cudaFree here would synchronise the whole device, i.e. wait for
        // the other virtual ranks' kernels -- which, with the fused peer exchange, may be waiting
        // for this rank's next kernels (deadlock)
        const size_t need = es * (size_t)std::max<int64_t>(count, 1) * nranks;
        if (scratch_.bytes() < need) scratch_.alloc(std::max(need, (size_t)4096));
        DevBuf& tmp = scratch_;
        for (int q = 0; q < nranks; ++q)
            if (count > 0)
                MX_CUDA(cudaMemcpyAsync(static_cast<char*>(tmp.get()) + q * count * es, g_->posts[q].buf, count * es,
                                        cudaMemcpyDeviceToDevice, st));
        MX_CUDA(cudaStreamSynchronize(st));
        g_->barrier();  // every rank has read every buffer before anyone overwrites its own
        if (count > 0) {
            const unsigned blocks = (unsigned)std::min<int64_t>(1024, ceil_div(count, 256));
            switch (t) {
                case DType::I32: sum_ranks_kernel<<<blocks, 256, 0, st>>>(tmp.as<int32_t>(), nranks, count, (int32_t*)buf); break;
                case DType::I64: sum_ranks_kernel<<<blocks, 256, 0, st>>>(tmp.as<int64_t>(), nranks, count, (int64_t*)buf); break;
                case DType::F32: sum_ranks_kernel<<<blocks, 256, 0, st>>>(tmp.as<float>(), nranks, count, (float*)buf); break;
                case DType::F64: sum_ranks_kernel<<<blocks, 256, 0, st>>>(tmp.as<double>(), nranks, count, (double*)buf); break;
            }
            MX_LAUNCHED();
        }
        MX_CUDA(cudaStreamSynchronize(st));
    }

    void reduce_scatter_sum(const void* send, void* recv, int64_t count, DType t, cudaStream_t st) override {
        MX_CUDA(cudaStreamSynchronize(st));
        const size_t es = dtype_size(t);
        g_->posts[rank].send = send;
        g_->barrier();
        const size_t need = es * (size_t)std::max<int64_t>(count, 1) * nranks;
        if (scratch_.bytes() < need) scratch_.alloc(std::max(need, (size_t)4096));
        for (int q = 0; q < nranks; ++q)
            if (count > 0)
                MX_CUDA(cudaMemcpyAsync(static_cast<char*>(scratch_.get()) + q * count * es,
                                        static_cast<const char*>(g_->posts[q].send) + rank * count * es, count * es,
                                        cudaMemcpyDeviceToDevice, st));
        MX_CUDA(cudaStreamSynchronize(st));
        g_->barrier();  // every rank has read its block of every send buffer
        if (count > 0) {
            const unsigned blocks = (unsigned)std::min<int64_t>(1024, ceil_div(count, 256));
            switch (t) {
                case DType::F32: sum_ranks_kernel<<<blocks, 256, 0, st>>>(scratch_.as<float>(), nranks, count, (float*)recv); break;
                case DType::F64: sum_ranks_kernel<<<blocks, 256, 0, st>>>(scratch_.as<double>(), nranks, count, (double*)recv); break;
                default: fail(MEMXCT_ERR_UNSUPPORTED, "internal: integer reduce-scatter");
            }
            MX_LAUNCHED();
        }
        MX_CUDA(cudaStreamSynchronize(st));
    }

    void allgather(const void* send, void* recv, int64_t count, DType t, cudaStream_t st) override {
        MX_CUDA(cudaStreamSynchronize(st));
        const size_t es = dtype_size(t);
        g_->posts[rank].send = send;
        g_->barrier();
        for (int q = 0; q < nranks; ++q)
            if (count > 0)
                MX_CUDA(cudaMemcpyAsync(static_cast<char*>(recv) + q * count * es, g_->posts[q].send, count * es,
                                        cudaMemcpyDeviceToDevice, st));
        MX_CUDA(cudaStreamSynchronize(st));
        g_->barrier();
    }

    void alltoallv(const void* send, const int64_t* scount, const int64_t* sdispl, void* recv,
                   const int64_t* rcount, const int64_t* rdispl, DType t, cudaStream_t st) override {
        MX_CUDA(cudaStreamSynchronize(st));
        const size_t es = dtype_size(t);
        auto& me = g_->posts[rank];
        me.send = send;
        me.sdispl = sdispl;
        me.scount = scount;
        g_->barrier();
        for (int q = 0; q < nranks; ++q) {
            const auto& pq = g_->posts[q];
            if (pq.scount[rank] != rcount[q]) fail(MEMXCT_ERR_CUDA, "internal: all-to-allv count mismatch");
            if (rcount[q] > 0)
                MX_CUDA(cudaMemcpyAsync(static_cast<char*>(recv) + rdispl[q] * es,
                                        static_cast<const char*>(pq.send) + pq.sdispl[rank] * es, rcount[q] * es,
                                        cudaMemcpyDeviceToDevice, st));
        }
        MX_CUDA(cudaStreamSynchronize(st));
        g_->barrier();
    }

    std::vector<int64_t> allgather_host(int64_t v, cudaStream_t st) override {
        g_->posts[rank].value = v;
        g_->barrier();
        std::vector<int64_t> out(nranks);
        for (int q = 0; q < nranks; ++q) out[q] = g_->posts[q].value;
        g_->barrier();
        return out;
    }

    std::vector<int64_t> allgather_vec(const std::vector<int64_t>& v, cudaStream_t st) override {
        g_->posts[rank].vec = &v;
        g_->barrier();
        std::vector<int64_t> out;
        for (int q = 0; q < nranks; ++q) out.insert(out.end(), g_->posts[q].vec->begin(), g_->posts[q].vec->end());
        g_->barrier();
        return out;
    }

    std::vector<void*> map_peers(void* local, cudaStream_t st) override {
        g_->posts[rank].buf = local;  // same device, same process: plain pointers
        g_->barrier();
        std::vector<void*> out(nranks);
        for (int q = 0; q < nranks; ++q) out[q] = g_->posts[q].buf;
        g_->barrier();
        return out;
    }

private:
    std::shared_ptr<LocalGroup> g_;
    DevBuf scratch_;
};

}  // namespace

std::unique_ptr<Comm> make_local_comm(std::shared_ptr<LocalGroup> g, int rank) {
    return std::make_unique<LocalComm>(std::move(g), rank);
}

}  // namespace mx
