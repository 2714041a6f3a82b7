// peer.cu -- fused compute + exchange over peer memory (the "overlapped
// interactions" of P:744-756 and the C step of A = R C A_p), EXCHANGE = 1.
//
// Instead of SpMV -> all-to-allv (NCCL) -> reduce, each rank maps its peers' receive buffers,
// footprint buffers and flag arrays into its address space (CUDA IPC over NVLink for NCCL ranks,
// plain pointers for virtual ranks) and:
//   forward  the SpMV epilogue stores every footprint row's partial directly into its owner's
//            receive buffer and publishes an epoch flag (spmv.cu: remote_epilogue); the owner
//            waits for every peer's flag and reduces (R) in fixed peer order;
//   back     the owner's pack kernel stores its ray values directly into every interacting
//            rank's footprint buffer (R^T and C^T in one kernel) and publishes a flag; each rank
//            waits for all owners, then runs A_p^T.
// Credit flags make buffer reuse safe for any call sequence: a rank writes into a peer's buffer
// only after that peer has finished consuming the previous contents.  All waits are one-thread
// kernels (a spinning CTA never blocks a co-resident rank's kernels), with a time-out that sets
// the process's abort word and returns instead of hanging (plan.h: peer_abort_word).
#include "plan.h"

namespace mx {

namespace {

constexpr int kT = 256;

__device__ __forceinline__ void st_release(unsigned long long* p, unsigned long long v) { st_release_sys(p, v); }

// wait until flags[base + q] >= flags[target_index] for every q < P
__global__ void wait_kernel(const unsigned long long* flags, int P, int base, int target_index, int me,
                            unsigned int* abort) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    wait_flags(flags, base, P, ld_acquire_sys(flags + target_index), me, abort);
}

// peer_flags[q][slot] = flags[value_index] for every q (credit: "done with what you sent me")
struct SignalArgs {
    unsigned long long* flag[kMaxPeers];
};
__global__ void signal_kernel(SignalArgs sa, int P, int slot, const unsigned long long* flags, int value_index) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const unsigned long long v = flags[value_index];
    __threadfence_system();
    for (int q = 0; q < P; ++q) st_release(sa.flag[q] + slot, v);
}

__global__ void publish_epoch_kernel(SignalArgs sa, int P, int slot, unsigned long long* flags, int epoch_index) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    __threadfence_system();
    const unsigned long long e = flags[epoch_index] + 1;
    flags[epoch_index] = e;
    for (int q = 0; q < P; ++q) st_release(sa.flag[q] + slot, e);
}

// R^T + C^T: value j (recv order, peer g = the range containing j) goes to g's footprint buffer
// (pa.fold: thread 0 of every CTA first waits for the peers' credits -- footprint buffers
// consumed -- reading the epoch before this CTA's ticket, i.e. before the last CTA bumps it).
// Each CTA packs one contiguous range of the recv order, so only CTAs whose range reaches
// another rank's slice pay a system-scope fence; the others' stores stay on this GPU (own
// footprint slice) and a device-scope fence orders them before the ticket.
__global__ void pack_remote_kernel(const float* __restrict__ y, const int32_t* __restrict__ idx, int64_t n,
                                   PeerArgs pa) {
    __shared__ bool am_last;
    if (pa.fold) {
        if (threadIdx.x == 0)
            wait_flags(pa.my_flags, pa.wait_base, pa.P, pa.my_flags[pa.epoch_index], pa.me, pa.abort);
        __syncthreads();
    }
    // destination table in shared memory (no dynamic indexing of the kernel parameters)
    __shared__ int64_t bound[kMaxPeers + 1], off[kMaxPeers];
    __shared__ float* dst[kMaxPeers];
    if (threadIdx.x <= (unsigned)pa.P) bound[threadIdx.x] = pa.bound[threadIdx.x];
    if (threadIdx.x < (unsigned)pa.P) {
        dst[threadIdx.x] = pa.dst[threadIdx.x];
        off[threadIdx.x] = pa.off[threadIdx.x];
    }
    __syncthreads();
    const int64_t per = (n + gridDim.x - 1) / gridDim.x;
    const int64_t chunk = (per + blockDim.x - 1) / blockDim.x * blockDim.x;
    const int64_t j0 = (int64_t)blockIdx.x * chunk, j1 = min(n, j0 + chunk);
    int g = 0;
    while (g + 1 < pa.P && j0 + (int64_t)threadIdx.x >= bound[g + 1]) ++g;
    constexpr int kU = 4;  // independent (index, value) loads in flight per thread
    for (int64_t j = j0 + threadIdx.x; j < j1; j += kU * (int64_t)blockDim.x) {
        float v[kU];
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t jj = j + u * (int64_t)blockDim.x;
            v[u] = jj < j1 ? y[idx[jj]] : 0.f;
        }
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int64_t jj = j + u * (int64_t)blockDim.x;
            if (jj >= j1) break;
            while (g + 1 < pa.P && jj >= bound[g + 1]) ++g;   // ranges ascend with j
            dst[g][off[g] + jj] = v[u];
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        const bool remote = j0 < j1 && (j0 < pa.bound[pa.me] || j1 > pa.bound[pa.me + 1]);
        if (remote) __threadfence_system();
        else __threadfence();
        am_last = (atomicAdd(pa.ticket, 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (!am_last || threadIdx.x != 0) return;
    __threadfence_system();
    const unsigned long long e = pa.my_flags[pa.epoch_index] + 1;
    pa.my_flags[pa.epoch_index] = e;
    for (int g = 0; g < pa.P; ++g) st_release(pa.flag[g] + pa.slot + pa.me, e);
    *pa.ticket = 0u;
}

// CG dot products over peer memory (EXCHANGE = 1): the B200-native form of the two fp64
// allreduces per CG iteration, which on NVSwitch cost a collective launch each
// (~10-20 us) against a per-rank SpMV pair of ~0.5 ms at P = 8 (config 3).  One thread: bump my
// epoch e; store my K values into every rank's slot [e & 1][me] (peer stores over NVLink), fence,
// publish e to every rank's arrival flag [me]; wait until every rank's flag in my array reaches e;
// sum the P slots in rank order (rank 0's value first: the same fp64 additions on every rank, and
// the same as the virtual-rank transport's sum).  Two parity slots suffice: a rank can write epoch
// e + 2 into slot e & 1 only after it has seen every rank's epoch e + 1 arrival, which each rank
// publishes after it has read its epoch-e slots.
struct DotArgs {
    double* dst[kMaxPeers];              // rank q's value array (peer pointer)
    unsigned long long* flag[kMaxPeers];  // rank q's flag array (peer pointer)
    const double* mine;                  // my value array
    unsigned long long* my_flags;        // my flag array: [P arrivals | epoch]
};
__global__ void peer_allreduce_kernel(DotArgs da, int P, int me, double* v, int K, int64_t stride,
                                      unsigned int* abort) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const unsigned long long e = da.my_flags[P] + 1;
    da.my_flags[P] = e;
    const int par = (int)(e & 1ull);
    for (int q = 0; q < P; ++q)
        for (int s = 0; s < K; ++s) da.dst[q][((int64_t)par * P + me) * kMaxDotSlices + s] = v[s * stride];
    __threadfence_system();
    for (int q = 0; q < P; ++q) st_release(da.flag[q] + me, e);
    wait_flags(da.my_flags, 0, P, e, me, abort);
    for (int s = 0; s < K; ++s) {
        const volatile double* m = da.mine + (int64_t)par * P * kMaxDotSlices + s;
        double acc = m[0];
        for (int q = 1; q < P; ++q) acc += m[(int64_t)q * kMaxDotSlices];
        v[s * stride] = acc;
    }
}

unsigned nblocks(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, kT), 4 * num_sms())); }

SignalArgs signal_args(const Plan& P) {
    SignalArgs sa{};
    for (int q = 0; q < P.nranks; ++q) sa.flag[q] = static_cast<unsigned long long*>(P.ex.peer_flags[q]);
    return sa;
}

}  // namespace

unsigned int* peer_abort_word() {
    static unsigned int* word = [] {
        void* p = nullptr;
        MX_CUDA(cudaHostAlloc(&p, sizeof(unsigned int), cudaHostAllocMapped | cudaHostAllocPortable));
        *static_cast<volatile unsigned int*>(p) = 0u;
        void* d = nullptr;
        MX_CUDA(cudaHostGetDevicePointer(&d, p, 0));
        return static_cast<unsigned int*>(d);  // = p under unified addressing
    }();
    return word;
}

void check_peer_abort() {
    if (*static_cast<volatile unsigned int*>(peer_abort_word()))
        fail(MEMXCT_ERR_NCCL, "a peer-exchange wait timed out on the device (a peer rank is gone); results of "
                              "the interrupted call are undefined");
}

void peer_setup(Plan& P, cudaStream_t st) {
    Exchange& X = P.ex;
    const int np = P.nranks;
    // Load every kernel of the fused path now: with lazy module loading the first launch of a
    // kernel can wait for the device, i.e. for a peer-flag wait that is spinning -- a deadlock.
    {
        cudaFuncAttributes fa;
        MX_CUDA(cudaFuncGetAttributes(&fa, wait_kernel));
        MX_CUDA(cudaFuncGetAttributes(&fa, signal_kernel));
        MX_CUDA(cudaFuncGetAttributes(&fa, publish_epoch_kernel));
        MX_CUDA(cudaFuncGetAttributes(&fa, pack_remote_kernel));
        MX_CUDA(cudaFuncGetAttributes(&fa, peer_allreduce_kernel));
        preload_exchange_kernels();
    }
    if (np > kMaxPeers) fail(MEMXCT_ERR_UNSUPPORTED, "fused peer exchange supports up to 16 ranks");
    if (P.esize != 4) fail(MEMXCT_ERR_UNSUPPORTED, "fused peer exchange is FP32 only");
    Comm& C = *P.comm;
    X.flags.alloc(4 * np + 2);
    MX_CUDA(cudaMemsetAsync(X.flags.p(), 0, 8 * (4 * np + 2), st));
    // folded waits only where every rank has its own GPU (see PeerArgs::fold); MEMXCT_PEER_FOLD=0/1
    X.fold = !C.shares_device();
    if (const char* e = std::getenv("MEMXCT_PEER_FOLD")) X.fold = e[0] == '1';
    MX_CUDA(cudaStreamSynchronize(st));
    // where my rows land in every owner's receive buffer, and my values in every peer's footprint
    std::vector<int64_t> rd(X.rdispl.begin(), X.rdispl.end()), sd(X.sdispl.begin(), X.sdispl.end());
    const auto all_rd = C.allgather_vec(rd, st);  // [q][np + 1]
    const auto all_sd = C.allgather_vec(sd, st);
    X.fwd_off.assign(np, 0);
    X.back_off.assign(np, 0);
    for (int h = 0; h < np; ++h) X.fwd_off[h] = all_rd[h * (np + 1) + P.rank] - X.sdispl[h];
    for (int g = 0; g < np; ++g) X.back_off[g] = all_sd[g * (np + 1) + P.rank] - X.rdispl[g];
    X.peer_recv = C.map_peers(X.recv_buf.get(), st);
    X.peer_yfp = C.map_peers(X.y_fp.get(), st);
    X.peer_flags = C.map_peers(X.flags.p(), st);
    X.dotx.alloc(2 * (int64_t)np * kMaxDotSlices);
    X.dflags.alloc(np + 1);
    MX_CUDA(cudaMemsetAsync(X.dflags.p(), 0, 8 * (np + 1), st));
    MX_CUDA(cudaStreamSynchronize(st));
    X.peer_dotx = C.map_peers(X.dotx.p(), st);
    X.peer_dflags = C.map_peers(X.dflags.p(), st);
    X.peer = true;
}

namespace {
PeerArgs base_args(const Plan& P) {
    PeerArgs pa;
    pa.P = P.nranks;
    pa.me = P.rank;
    pa.my_flags = P.ex.flags.p();
    pa.fold = P.ex.fold ? 1 : 0;
    pa.abort = peer_abort_word();
    for (int q = 0; q < P.nranks; ++q) pa.flag[q] = static_cast<unsigned long long*>(P.ex.peer_flags[q]);
    return pa;
}
// the CG dot of this projection summed over the ranks inside its last kernel (fold mode only:
// a spinning last CTA on a GPU of its own never blocks a peer's kernels)
void set_dot_fold(const Plan& P, PeerArgs& pa) {
    const Exchange& X = P.ex;
    pa.dot_fold = 1;
    for (int q = 0; q < P.nranks; ++q) {
        pa.dot_dst[q] = static_cast<double*>(X.peer_dotx[q]);
        pa.dot_flag[q] = static_cast<unsigned long long*>(X.peer_dflags[q]);
    }
    pa.dot_mine = X.dotx.p();
    pa.dot_my_flags = X.dflags.p();
}
}  // namespace

// Flags of rank g ([4P + 2]): arrivals fwd [0, P) | arrivals back [P, 2P) | credits fwd [2P, 3P) |
// credits back [3P, 4P) | my fwd epoch 4P | my back epoch 4P + 1.
// Forward: (1) owners have consumed my previous partials (credits fwd >= my epoch); (2) A_p
// stores the partials into the owners' receive buffers; a one-thread kernel then bumps the epoch
// and publishes it to every owner; (3) every peer's partials for my rays have arrived; (4) R (+
// dot); (5) credits back to every peer.  Folded (NCCL ranks): (1) runs at the start of A_p's
// CTAs, (3) and (5) inside the reduction kernel.
void peer_forward(Plan& P, const float* x, float* y, double* dot_out, cudaStream_t st) {
    Exchange& X = P.ex;
    const int np = P.nranks;
    unsigned long long* fl = X.flags.p();
    // (1) credits: a one-thread wait kernel in both modes -- folded into A_p's CTAs, the
    // system-scope wait delayed every partition (+26 us per config-3 forward, r02j)
    wait_kernel<<<1, 32, 0, st>>>(fl, np, 2 * np, 4 * np, P.rank, peer_abort_word());
    MX_LAUNCHED();
    PeerArgs pa = base_args(P);
    pa.fold = 0;  // the credits are awaited above
    for (int h = 0; h <= np; ++h) pa.bound[h] = X.sdispl[h];
    for (int h = 0; h < np; ++h) {
        pa.dst[h] = static_cast<float*>(X.peer_recv[h]);
        pa.off[h] = X.fwd_off[h];
    }
    pa.ticket = X.tickets.p();
    pa.slot = 0;
    pa.epoch_index = 4 * np;
    pa.wait_base = 2 * np;
    spmv_f32_remote(P.fwd, x, pa, st);
    publish_epoch_kernel<<<1, 32, 0, st>>>(signal_args(P), np, 0 + P.rank, fl, 4 * np);  // arrivals fwd
    MX_LAUNCHED();
    if (!X.fold) {
        wait_kernel<<<1, 32, 0, st>>>(fl, np, 0, 4 * np, P.rank, peer_abort_word());
        MX_LAUNCHED();
    }
    PeerArgs ra = base_args(P);
    if (X.fold && dot_out) set_dot_fold(P, ra);
    ra.slot = 2 * np;          // credits fwd in the senders' arrays
    ra.epoch_index = 4 * np;
    ra.wait_base = 0;          // arrivals fwd
    reduce_partials(P, X.recv_buf.as<float>(), y, dot_out, ra, st);
    if (!X.fold) {
        signal_kernel<<<1, 32, 0, st>>>(signal_args(P), np, 2 * np + P.rank, fl, 4 * np);
        MX_LAUNCHED();
    }
}

// Back: (1) every peer has finished reading my previous values from its footprint buffer
// (credits back); (2) R^T + C^T: the owned ray values stored straight into the peers' footprint
// buffers, last CTA publishes the back epoch; (3) every owner's values for my footprint have
// arrived; (4) A_p^T (+ dot); (5) credits to every peer (one-thread kernel).  Folded: (1) in the
// pack kernel's prologue, (3) in A_p^T's prologue.
void peer_back(Plan& P, const float* y, float* x, double* dot_out, cudaStream_t st) {
    Exchange& X = P.ex;
    const int np = P.nranks;
    unsigned long long* fl = X.flags.p();
    if (!X.fold) {
        wait_kernel<<<1, 32, 0, st>>>(fl, np, 3 * np, 4 * np + 1, P.rank, peer_abort_word());
        MX_LAUNCHED();
    }
    PeerArgs pa = base_args(P);
    for (int g = 0; g <= np; ++g) pa.bound[g] = X.rdispl[g];
    for (int g = 0; g < np; ++g) {
        pa.dst[g] = static_cast<float*>(X.peer_yfp[g]);
        pa.off[g] = X.back_off[g];
    }
    pa.ticket = X.tickets.p() + 1;
    pa.slot = np;
    pa.epoch_index = 4 * np + 1;
    pa.wait_base = 3 * np;
    pack_remote_kernel<<<nblocks(X.nrecv), kT, 0, st>>>(y, X.recv_idx.p(), X.nrecv, pa);
    MX_LAUNCHED();
    if (!X.fold) {
        wait_kernel<<<1, 32, 0, st>>>(fl, np, np, 4 * np + 1, P.rank, peer_abort_word());
        MX_LAUNCHED();
    }
    PeerArgs ba = base_args(P);
    if (X.fold && dot_out) set_dot_fold(P, ba);
    ba.ticket = X.tickets.p() + 3;
    ba.slot = 3 * np;          // credits back in the owners' arrays
    ba.epoch_index = 4 * np + 1;
    ba.wait_base = np;         // arrivals back
    spmv_f32_peer_back(P.back, X.y_fp.as<float>(), x, dot_out ? X.dot_part.p() : nullptr, dot_out,
                       X.tickets.p() + 4, ba, st);
    // credits to every peer (footprint buffer consumed), after the kernel boundary
    signal_kernel<<<1, 32, 0, st>>>(signal_args(P), np, 3 * np + P.rank, fl, 4 * np + 1);
    MX_LAUNCHED();
}

void peer_allreduce(Plan& P, double* v, int K, int64_t stride, cudaStream_t st) {
    if (K < 1) return;
    if (K > kMaxDotSlices) fail(MEMXCT_ERR_INVALID_ARG, "peer dot: more than 64 slices");
    Exchange& X = P.ex;
    DotArgs da{};
    for (int q = 0; q < P.nranks; ++q) {
        da.dst[q] = static_cast<double*>(X.peer_dotx[q]);
        da.flag[q] = static_cast<unsigned long long*>(X.peer_dflags[q]);
    }
    da.mine = X.dotx.p();
    da.my_flags = X.dflags.p();
    peer_allreduce_kernel<<<1, 32, 0, st>>>(da, P.nranks, P.rank, v, K, stride, peer_abort_word());
    MX_LAUNCHED();
}

}  // namespace mx
