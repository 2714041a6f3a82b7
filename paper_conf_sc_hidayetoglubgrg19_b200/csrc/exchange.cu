// exchange.cu -- domain decomposition over P GPUs (sec. 3.4, Table 1):
//   a3  both domains split into contiguous Hilbert tile ranges balanced on nonzeros;
//   a6  exchange maps of the sparse communication;
//   a8  forward  y = R C A_p x: partial projection on the footprint rays, all-to-allv of the
//       partials to the ray owners, reduction in fixed peer order;
//   a9  back     x = A_p^T C^T R^T y: owners duplicate their ray values to every interacting
//       rank (the transposed communication), then the partial backprojection.
// The footprint rays of a rank are kept in Hilbert order; since ray ownership is a contiguous
// Hilbert range, that is also (owner, Hilbert) order, so the forward partials bound for each
// owner are one contiguous slice of the SpMV output (zero-copy send), and the backprojection
// receives straight into the same slices.
#include <cub/device/device_segmented_reduce.cuh>

#include <algorithm>
#include <vector>

#include "comm.h"
#include "plan.h"

namespace mx {

std::vector<int64_t> partition_ranges(const std::vector<int64_t>& w, int32_t parts) {
    const int64_t k = (int64_t)w.size();
    std::vector<int64_t> pre(k + 1, 0);
    for (int64_t i = 0; i < k; ++i) pre[i + 1] = pre[i] + w[i];
    const int64_t total = pre[k];
    std::vector<int64_t> b(parts + 1, 0);
    b[parts] = k;
    for (int32_t g = 1; g < parts; ++g) {
        // first boundary whose prefix reaches g/P of the total (ties: the nearer of the two)
        const int64_t target = (int64_t)((long double)total * g / parts + 0.5L);
        int64_t i = std::lower_bound(pre.begin(), pre.end(), target) - pre.begin();
        if (i > 0 && i <= k && (target - pre[i - 1]) < (pre[i] - target)) --i;
        i = std::max(i, b[g - 1]);
        if (k >= parts) i = std::max<int64_t>(i, b[g - 1] + 1);       // every rank gets a tile
        if (k >= parts) i = std::min<int64_t>(i, k - (parts - g));
        b[g] = std::min(i, k);
    }
    return b;
}

namespace {

constexpr int kT = 256;

unsigned nblocks(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, kT), 1 << 20)); }

// grid of the reduction R and the packs R^T: 8 CTAs of kT threads per SM, kRedU elements per thread
// per pass (one element per thread over ~6000 CTAs ran the config-3 reduction at ~1.3 TB/s)
constexpr int kRedU = 4;
unsigned red_blocks(int64_t n) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, (int64_t)kT * kRedU), 8 * num_sms()));
}

std::vector<int64_t> to_host_i64(const int64_t* d, int64_t n, cudaStream_t st) {
    std::vector<int64_t> h(n);
    MX_CUDA(cudaMemcpyAsync(h.data(), d, 8 * n, cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    return h;
}

// R: owned ray i = its received partials added in peer order (reduction-map CSR ptr / pos;
// ptr == nullptr: y[i] = recv[i], the dense exchange's owned block).  Optionally the CG dot
// <y, y> of the owned rays: per-CTA fixed tree, the last CTA (ticket) adds the CTA partials in
// CTA order -- deterministic, and the same sums for every exchange (same grid, same values).
// pa.fold (fused exchange on NCCL ranks, peer.cu): thread 0 of every CTA first waits for every
// peer's arrival flag, and the last CTA returns the credits (receive buffer consumed).
template <class T>
__global__ void __launch_bounds__(kT)
reduce_dot_kernel(const T* __restrict__ recv, const int64_t* __restrict__ ptr, const int32_t* __restrict__ pos,
                  int64_t nown, T* __restrict__ y, double* part, double* dot_out, unsigned int* ticket, PeerArgs pa,
                  const T* __restrict__ self, int64_t self_lo, int64_t self_hi) {
    __shared__ double red[kT / 32];
    __shared__ bool am_last;
    if (pa.fold) {
        if (threadIdx.x == 0)
            wait_flags(pa.my_flags, pa.wait_base, pa.P, pa.my_flags[pa.epoch_index], pa.me, pa.abort);
        __syncthreads();
    }
    double d = 0.0;
    // kRedU independent owned rays per thread per pass (a fixed element -> thread map, so the
    // dot's summation order depends only on the grid)
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i0 < nown; i0 += kRedU * stride) {
#pragma unroll
        for (int u = 0; u < kRedU; ++u) {
            const int64_t i = i0 + u * stride;
            if (i >= nown) break;
            T acc;
            if (ptr) {
                acc = T(0);
                for (int64_t k = ptr[i]; k < ptr[i + 1]; ++k) {  // peer order
                    const int64_t q = pos[k];
                    // this rank's own partial is read in place from its footprint slice (`self`):
                    // no copy into the receive buffer
                    acc += (q >= self_lo && q < self_hi) ? self[q - self_lo] : recv[q];
                }
            } else {
                acc = recv[i];
            }
            y[i] = acc;
            d += (double)acc * (double)acc;
        }
    }
    if (!dot_out && !pa.fold) return;
    if (dot_out) {
        for (int o = 16; o; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
        if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = d;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (dot_out) {
            double t = 0.0;
            for (int w = 0; w < kT / 32; ++w) t += red[w];
            part[blockIdx.x] = t;
        }
        __threadfence();
        am_last = (atomicAdd(ticket, 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (!am_last) return;
    __threadfence();
    if (dot_out) {  // the last CTA adds the CTA partials: strided per thread, then the fixed tree
        double t = 0.0;
        for (unsigned b = threadIdx.x; b < gridDim.x; b += blockDim.x) t += ((volatile double*)part)[b];
        for (int o = 16; o; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
        __syncthreads();
        if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = t;
        __syncthreads();
        if (threadIdx.x == 0) {
            double tot = 0.0;
            for (int w = 0; w < kT / 32; ++w) tot += red[w];
            *dot_out = tot;
        }
    }
    if (threadIdx.x != 0) return;
    if (pa.fold) {
        __threadfence_system();
        const unsigned long long e = pa.my_flags[pa.epoch_index];
        for (int q = 0; q < pa.P; ++q) st_release_sys(pa.flag[q] + pa.slot + pa.me, e);
        // the CG dot over the ranks (credits are out first: peers may be waiting on them)
        if (dot_out && pa.dot_fold) peer_dot_allreduce(pa, dot_out);
    }
    *ticket = 0u;
}

template <class T>
__global__ void pack_kernel(const T* __restrict__ y, const int32_t* __restrict__ idx, int64_t n, T* __restrict__ out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = y[idx[i]];
}

// R^T with the self slice [lo, hi) of the pack order written straight into this rank's
// footprint slice `self` (no copy through the receive buffer and the all-to-allv)
template <class T>
__global__ void pack_self_kernel(const T* __restrict__ y, const int32_t* __restrict__ idx, int64_t n,
                                 T* __restrict__ out, T* __restrict__ self, int64_t lo, int64_t hi) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i0 < n; i0 += kRedU * stride) {
#pragma unroll
        for (int u = 0; u < kRedU; ++u) {
            const int64_t i = i0 + u * stride;
            if (i >= n) break;
            const T v = y[idx[i]];
            if (i >= lo && i < hi) self[i - lo] = v;
            else out[i] = v;
        }
    }
}

template <class T>
__global__ void scatter_dense_kernel(const T* __restrict__ yfp, const int32_t* __restrict__ pos, int64_t n,
                                     T* __restrict__ dense) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dense[pos[i]] = yfp[i];
}

__global__ void flag_kernel(const int32_t* __restrict__ len, int64_t n, int32_t* __restrict__ flag) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        flag[i] = len[i] > 0;
}

__global__ void compact_kernel(const int32_t* __restrict__ len, const int64_t* __restrict__ pos, int64_t n,
                               int32_t* __restrict__ fp_rays, int32_t* __restrict__ fp_len) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (len[i] > 0) {
            fp_rays[pos[i]] = (int32_t)i;
            fp_len[pos[i]] = len[i];
        }
}

std::vector<int64_t> tile_sums(const int32_t* w, const std::vector<int64_t>& tile_off, cudaStream_t st) {
    const int64_t nt = (int64_t)tile_off.size() - 1;
    DevArr<int64_t> off, out;
    off.alloc(nt + 1);
    out.alloc(nt);
    MX_CUDA(cudaMemcpyAsync(off.p(), tile_off.data(), 8 * (nt + 1), cudaMemcpyHostToDevice, st));
    size_t tb = 0;
    MX_CUDA(cub::DeviceSegmentedReduce::Sum(nullptr, tb, w, out.p(), nt, off.p(), off.p() + 1, st));
    DevBuf tmp(tb);
    MX_CUDA(cub::DeviceSegmentedReduce::Sum(tmp.get(), tb, w, out.p(), nt, off.p(), off.p() + 1, st));
    MX_LAUNCHED();
    std::vector<int64_t> h(nt);
    MX_CUDA(cudaMemcpyAsync(h.data(), out.p(), 8 * nt, cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    return h;
}

}  // namespace

// a3: tomogram and sinogram ranges of this rank
void decompose(Plan& P, const Geometry& G, cudaStream_t st) {
    const int64_t npix = (int64_t)P.n * P.n, nrays = (int64_t)P.m * P.c;
    if (!P.dist) {
        P.t0 = 0; P.t1 = npix; P.s0 = 0; P.s1 = nrays;
        P.tomo_bounds = {0, npix};
        P.sino_bounds = {0, nrays};
        return;
    }
    // per-pixel nonzeros (column counts of A): each rank traces 1/P of the rays, then allreduce
    // (a shard probe has no peers: it traces every ray itself, the same counts)
    DevArr<int32_t> hist;
    hist.alloc(npix);
    MX_CUDA(cudaMemsetAsync(hist.p(), 0, 4 * npix, st));
    const int64_t ra = P.shard ? 0 : nrays * P.rank / P.nranks;
    const int64_t rb = P.shard ? nrays : nrays * (P.rank + 1) / P.nranks;
    trace_hist(P, G, nullptr, ra, rb - ra, 0, 0, false, hist.p(), st);
    if (!P.shard) P.comm->allreduce_sum(hist.p(), npix, DType::I32, st);
    const auto tw = tile_sums(hist.p(), P.tomo_tile_off, st);
    hist.reset();
    // per-ray nonzeros (row lengths of A)
    DevArr<int32_t> rl;
    rl.alloc(nrays);
    trace_count(P, G, nullptr, 0, nrays, 0, 0, false, rl.p(), st);
    const auto sw = tile_sums(rl.p(), P.sino_tile_off, st);
    const auto bt = partition_ranges(tw, P.nranks), bs = partition_ranges(sw, P.nranks);
    P.tomo_bounds.resize(P.nranks + 1);
    P.sino_bounds.resize(P.nranks + 1);
    for (int g = 0; g <= P.nranks; ++g) {
        P.tomo_bounds[g] = P.tomo_tile_off[bt[g]];
        P.sino_bounds[g] = P.sino_tile_off[bs[g]];
    }
    P.t0 = P.tomo_bounds[P.rank];
    P.t1 = P.tomo_bounds[P.rank + 1];
    P.s0 = P.sino_bounds[P.rank];
    P.s1 = P.sino_bounds[P.rank + 1];
}

// footprint rays of the local tomogram subdomain (all rays at P = 1) and their row lengths
int64_t footprint(Plan& P, const Geometry& G, DevArr<int32_t>& fp_len, cudaStream_t st) {
    const int64_t nrays = (int64_t)P.m * P.c;
    if (!P.dist) {
        fp_len.alloc(nrays);
        trace_count(P, G, nullptr, 0, nrays, 0, 0, false, fp_len.p(), st);
        P.fp_rays.reset();
        return nrays;
    }
    DevArr<int32_t> len;
    len.alloc(nrays);
    trace_count(P, G, nullptr, 0, nrays, P.t0, P.t1, true, len.p(), st);
    DevArr<int32_t> flag;
    DevArr<int64_t> flag64, pos;
    flag.alloc(nrays);
    flag64.alloc(nrays + 1);
    pos.alloc(nrays + 1);
    flag_kernel<<<nblocks(nrays), kT, 0, st>>>(len.p(), nrays, flag.p());
    MX_LAUNCHED();
    widen_i32_to_i64(flag.p(), flag64.p(), nrays, st);
    MX_CUDA(cudaMemsetAsync(flag64.p() + nrays, 0, 8, st));
    exclusive_scan_i64(flag64.p(), pos.p(), nrays + 1, st);
    int64_t nfp = 0;
    MX_CUDA(cudaMemcpyAsync(&nfp, pos.p() + nrays, 8, cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    P.fp_rays.alloc(std::max<int64_t>(nfp, 1));
    fp_len.alloc(std::max<int64_t>(nfp, 1));
    compact_kernel<<<nblocks(nrays), kT, 0, st>>>(len.p(), pos.p(), nrays, P.fp_rays.p(), fp_len.p());
    MX_LAUNCHED();
    MX_CUDA(cudaStreamSynchronize(st));
    return nfp;
}

// a6, receive side of a shard probe (no peers to ask): rank q's footprint slice bound for this
// owner is, in Hilbert order, every owned ray with a segment in q's pixel range [tomo_bounds[q],
// tomo_bounds[q+1]) -- exactly the rays q's own footprint pass selects.  Re-tracing the owned rays
// once per rank gives the counts (rcount) and owned-local indices (recv_idx) that the allgather and
// all-to-allv of build_exchange deliver on a real P-rank build.
void shard_receive_maps(Plan& P, const Geometry& G, cudaStream_t st) {
    Exchange& X = P.ex;
    const int np = P.nranks;
    const int64_t nown = P.s1 - P.s0;
    X.rcount.assign(np, 0);
    std::vector<int32_t> idx;
    std::vector<int32_t> len(std::max<int64_t>(nown, 1));
    DevArr<int32_t> dlen;
    dlen.alloc(std::max<int64_t>(nown, 1));
    for (int q = 0; q < np; ++q) {
        if (nown > 0) {
            trace_count(P, G, nullptr, P.s0, nown, P.tomo_bounds[q], P.tomo_bounds[q + 1], true, dlen.p(), st);
            MX_CUDA(cudaMemcpyAsync(len.data(), dlen.p(), 4 * nown, cudaMemcpyDeviceToHost, st));
            MX_CUDA(cudaStreamSynchronize(st));
        }
        const size_t before = idx.size();
        for (int64_t i = 0; i < nown; ++i)
            if (len[i] > 0) idx.push_back((int32_t)i);
        X.rcount[q] = (int64_t)(idx.size() - before);
    }
    X.recv_idx.alloc(std::max<int64_t>((int64_t)idx.size(), 1));
    if (!idx.empty())
        MX_CUDA(cudaMemcpy(X.recv_idx.p(), idx.data(), 4 * idx.size(), cudaMemcpyHostToDevice));
}

// Forward overlap of the sparse collective exchange (SURVEY 8(e) forward steps 1-2): the
// partitions of A_p are launched in two groups -- first every partition with a row owned by
// another rank, then (on a lower-priority side stream, concurrently) the partitions whose rows
// this rank owns itself -- so the all-to-allv of the remote slices starts while the self-owned
// rows are still being computed; the self slice is copied into the receive buffer after both.
// Launch order within each group: the layout's (partition order unless MEMXCT_PART_ORDER).
// MEMXCT_FWD_OVERLAP=0 disables it.
void setup_forward_overlap(Plan& P, cudaStream_t st) {
    Exchange& X = P.ex;
    Layout& L = P.fwd;
    if (const char* e = std::getenv("MEMXCT_FWD_OVERLAP"); e && e[0] == '0') return;
    const int64_t np = L.nparts;
    if (np == 0) return;
    const int64_t lo = X.sdispl[P.rank], hi = X.sdispl[P.rank + 1];  // my footprint slice
    const auto row0 = to_host_i64(L.prow0.p(), np + 1, st);
    std::vector<int32_t> pos(std::max<int64_t>(L.nrows, 1));
    if (L.out_idx.p() && L.nrows > 0)
        MX_CUDA(cudaMemcpy(pos.data(), L.out_idx.p(), 4 * L.nrows, cudaMemcpyDeviceToHost));
    else
        for (int64_t r = 0; r < L.nrows; ++r) pos[r] = (int32_t)r;
    std::vector<int32_t> cur(np);
    if (L.part_order.p()) MX_CUDA(cudaMemcpy(cur.data(), L.part_order.p(), 4 * np, cudaMemcpyDeviceToHost));
    else for (int64_t b = 0; b < np; ++b) cur[b] = (int32_t)b;
    std::vector<int32_t> first, second;
    for (int32_t p : cur) {
        bool self_only = true;
        for (int64_t r = row0[p]; r < row0[p + 1] && self_only; ++r) self_only = pos[r] >= lo && pos[r] < hi;
        (self_only ? second : first).push_back(p);
    }
    if (second.empty()) return;  // nothing to overlap
    first.insert(first.end(), second.begin(), second.end());
    L.part_order.alloc(np);
    MX_CUDA(cudaMemcpy(L.part_order.p(), first.data(), 4 * np, cudaMemcpyHostToDevice));
    L.n_first = np - (int64_t)second.size();
    int lo_prio = 0, hi_prio = 0;
    MX_CUDA(cudaDeviceGetStreamPriorityRange(&lo_prio, &hi_prio));
    MX_CUDA(cudaStreamCreateWithPriority(&X.side, cudaStreamNonBlocking, lo_prio));
    MX_CUDA(cudaEventCreateWithFlags(&X.ev_fork, cudaEventDisableTiming));
    MX_CUDA(cudaEventCreateWithFlags(&X.ev_join, cudaEventDisableTiming));
}

// a6: exchange maps (P > 1)
void build_exchange(Plan& P, cudaStream_t st) {
    if (!P.dist) return;
    Exchange& X = P.ex;
    const int np = P.nranks;
    std::vector<int32_t> fp(P.nfp);
    if (P.nfp > 0) MX_CUDA(cudaMemcpy(fp.data(), P.fp_rays.p(), 4 * P.nfp, cudaMemcpyDeviceToHost));
    X.sdispl.assign(np + 1, 0);
    for (int h = 0; h <= np; ++h)
        X.sdispl[h] = std::lower_bound(fp.begin(), fp.end(), (int32_t)std::min<int64_t>(P.sino_bounds[h], INT32_MAX)) - fp.begin();
    X.sdispl[np] = P.nfp;
    X.scount.assign(np, 0);
    for (int h = 0; h < np; ++h) X.scount[h] = X.sdispl[h + 1] - X.sdispl[h];
    if (!P.shard) {  // a shard probe has its rcount from shard_receive_maps
        X.rcount.assign(np, 0);
        for (int h = 0; h < np; ++h) {
            const auto v = P.comm->allgather_host(X.scount[h], st);  // v[q] = what rank q sends to owner h
            if (h == P.rank) X.rcount = v;
        }
    }
    X.rdispl.assign(np + 1, 0);
    for (int q = 0; q < np; ++q) X.rdispl[q + 1] = X.rdispl[q] + X.rcount[q];
    X.nrecv = X.rdispl[np];
    // index lists: owned-local index of each footprint ray, by owner
    std::vector<int32_t> idx(std::max<int64_t>(P.nfp, 1));
    for (int h = 0; h < np; ++h)
        for (int64_t i = X.sdispl[h]; i < X.sdispl[h + 1]; ++i) idx[i] = (int32_t)(fp[i] - P.sino_bounds[h]);
    if (!P.shard) {  // ... and its recv_idx
        DevArr<int32_t> send_idx;
        send_idx.alloc(std::max<int64_t>(P.nfp, 1));
        MX_CUDA(cudaMemcpy(send_idx.p(), idx.data(), 4 * P.nfp, cudaMemcpyHostToDevice));
        X.recv_idx.alloc(std::max<int64_t>(X.nrecv, 1));
        P.comm->alltoallv(send_idx.p(), X.scount.data(), X.sdispl.data(), X.recv_idx.p(), X.rcount.data(),
                          X.rdispl.data(), DType::I32, st);
        MX_CUDA(cudaStreamSynchronize(st));
    }
    // reduction map R: for every owned ray, its received partials in peer order (stable sort)
    const int64_t nown = P.s1 - P.s0;
    DevArr<uint32_t> keys_out, perm;
    keys_out.alloc(std::max<int64_t>(X.nrecv, 1));
    perm.alloc(std::max<int64_t>(X.nrecv, 1));
    if (X.nrecv > 0)
        stable_sort_by_key(reinterpret_cast<const uint32_t*>(X.recv_idx.p()), keys_out.p(), perm.p(), X.nrecv,
                           std::max<int64_t>(nown, 1), st);
    X.red_ptr.alloc(nown + 1);
    row_ptr_from_sorted(keys_out.p(), X.nrecv, nown, X.red_ptr.p(), st);
    X.red_pos.alloc(std::max<int64_t>(X.nrecv, 1));
    if (X.nrecv > 0)
        MX_CUDA(cudaMemcpyAsync(X.red_pos.p(), perm.p(), 4 * X.nrecv, cudaMemcpyDeviceToDevice, st));
    X.y_fp.alloc(P.esize * std::max<int64_t>(P.nfp, 1));
    X.recv_buf.alloc(P.esize * std::max<int64_t>(X.nrecv, 1));
    X.tickets.alloc(8);
    MX_CUDA(cudaMemsetAsync(X.tickets.p(), 0, 32, st));
    X.dot_part.alloc(std::max<int64_t>({P.back.nparts, (int64_t)red_blocks(nown), 8 * num_sms()}));
    if (P.opt.exchange == 0 && !P.shard) setup_forward_overlap(P, st);
    if (P.opt.exchange == 2) {  // dense collectives: footprint row i -> [owner][owned-local index]
        X.maxown = 0;
        for (int h = 0; h < np; ++h) X.maxown = std::max(X.maxown, P.sino_bounds[h + 1] - P.sino_bounds[h]);
        if ((int64_t)np * X.maxown >= INT32_MAX) fail(MEMXCT_ERR_UNSUPPORTED, "dense exchange: sinogram too large");
        std::vector<int32_t> dpos(std::max<int64_t>(P.nfp, 1));
        for (int h = 0; h < np; ++h)
            for (int64_t i = X.sdispl[h]; i < X.sdispl[h + 1]; ++i) dpos[i] = (int32_t)(h * X.maxown + idx[i]);
        X.dense_pos.alloc(std::max<int64_t>(P.nfp, 1));
        MX_CUDA(cudaMemcpy(X.dense_pos.p(), dpos.data(), 4 * std::max<int64_t>(P.nfp, 1), cudaMemcpyHostToDevice));
        X.dense_buf.alloc(P.esize * std::max<int64_t>(np * X.maxown, 1));
        X.dense_own.alloc(P.esize * std::max<int64_t>(X.maxown, 1));
        X.dense = true;
    }
    MX_CUDA(cudaStreamSynchronize(st));
    if (P.opt.exchange == 1) peer_setup(P, st);  // fused peer-memory exchange (peer.cu)
}

// self (nullable): this rank's footprint partials; the receive positions [rdispl[me],
// rdispl[me + 1]) are then read from self instead of `recv` (the self slice is not copied)
template <class T>
void launch_reduce_dot(Plan& P, const T* recv, bool csr, T* y, double* dot_out, const PeerArgs& pa, cudaStream_t st,
                       const T* self = nullptr) {
    Exchange& X = P.ex;
    const int64_t nown = P.s1 - P.s0;
    const int64_t lo = self ? X.rdispl[P.rank] : 0, hi = self ? X.rdispl[P.rank + 1] : 0;
    reduce_dot_kernel<T><<<red_blocks(nown), kT, 0, st>>>(recv, csr ? X.red_ptr.p() : nullptr, X.red_pos.p(), nown, y,
                                                       X.dot_part.p(), dot_out, X.tickets.p() + 2, pa, self, lo, hi);
    MX_LAUNCHED();
}

// the all-to-allv counts without this rank's own slice (it stays in place, see above)
struct RemoteCounts {
    std::vector<int64_t> sc, rc;
    RemoteCounts(const Exchange& X, int me) : sc(X.scount), rc(X.rcount) { sc[me] = rc[me] = 0; }
};

// Forward communication: footprint partials `yfp` (nfp) -> owned ray values `yown` (nown).
// Sparse (default): C = all-to-allv of the per-owner slices into `rb` (nrecv), R = per owned ray
// the received partials added in peer order.  Dense (EXCHANGE = 2): the partials scattered into a
// zeroed [P][maxown] sinogram, reduce-scatter (rank g receives block g summed over the ranks).
template <class T>
static void exchange_fwd(Plan& P, const T* yfp, T* rb, T* yown, cudaStream_t st, double* dot_out = nullptr) {
    Exchange& X = P.ex;
    const DType t = sizeof(T) == 4 ? DType::F32 : DType::F64;
    const int64_t nown = P.s1 - P.s0;
    if (X.dense) {
        T* d = X.dense_buf.as<T>();
        MX_CUDA(cudaMemsetAsync(d, 0, sizeof(T) * (size_t)(P.nranks * X.maxown), st));
        if (P.nfp > 0) {
            scatter_dense_kernel<T><<<nblocks(P.nfp), kT, 0, st>>>(yfp, X.dense_pos.p(), P.nfp, d);
            MX_LAUNCHED();
        }
        P.comm->reduce_scatter_sum(d, X.dense_own.get(), X.maxown, t, st);
        launch_reduce_dot<T>(P, X.dense_own.as<T>(), false, yown, dot_out, PeerArgs{}, st);  // copy (+ dot)
        return;
    }
    const RemoteCounts rcnt(X, P.rank);
    P.comm->alltoallv(yfp, rcnt.sc.data(), X.sdispl.data(), rb, rcnt.rc.data(), X.rdispl.data(), t, st);  // C
    launch_reduce_dot<T>(P, rb, true, yown, dot_out, PeerArgs{}, st, yfp + X.sdispl[P.rank]);            // R
}

// Back communication: owned ray values `yown` -> every footprint ray's value in `yfp`.  Sparse:
// R^T = pack of the owned values each peer needs (recv order) into `rb`, C^T = the reverse
// all-to-allv straight into the footprint slices.  Dense: allgather of the owned values into the
// [P][maxown] sinogram, gather of the footprint rays.
template <class T>
static void exchange_back(Plan& P, const T* yown, T* rb, T* yfp, cudaStream_t st, bool prepacked = false) {
    Exchange& X = P.ex;
    const DType t = sizeof(T) == 4 ? DType::F32 : DType::F64;
    if (X.dense) {
        const int64_t nown = P.s1 - P.s0;
        if (nown > 0)
            MX_CUDA(cudaMemcpyAsync(X.dense_own.get(), yown, sizeof(T) * nown, cudaMemcpyDeviceToDevice, st));
        P.comm->allgather(X.dense_own.get(), X.dense_buf.get(), X.maxown, t, st);
        if (P.nfp > 0) {
            pack_kernel<T><<<nblocks(P.nfp), kT, 0, st>>>(X.dense_buf.as<T>(), X.dense_pos.p(), P.nfp, yfp);
            MX_LAUNCHED();
        }
        return;
    }
    if (X.nrecv > 0 && !prepacked) {  // R^T (own slice straight into the footprint buffer)
        pack_self_kernel<T><<<red_blocks(X.nrecv), kT, 0, st>>>(yown, X.recv_idx.p(), X.nrecv, rb, yfp + X.sdispl[P.rank],
                                                             X.rdispl[P.rank], X.rdispl[P.rank + 1]);
        MX_LAUNCHED();
    }
    const RemoteCounts rcnt(X, P.rank);
    P.comm->alltoallv(rb, rcnt.rc.data(), X.rdispl.data(), yfp, rcnt.sc.data(), X.sdispl.data(), t, st);  // C^T
}

// P > 1 with dot_out: the CG dot of the rank's output part is fused into the reduction
// (forward) or into A_p^T's epilogue (back, per-partition tree + last-CTA sum); the caller sums
// it over the ranks.
template <class T>
static void forward_t(Plan& P, const T* x, T* y, double* dot_out, cudaStream_t st) {
    if (!P.dist) {
        spmv_any(P, P.fwd, x, y, st);
        return;
    }
    Exchange& X = P.ex;
    T* yfp = X.y_fp.as<T>();
    if (X.side && !X.dense) {  // overlap: remote-owned partitions, then C while the self-owned ones run
        const Layout& L = P.fwd;
        T* rb = X.recv_buf.as<T>();
        const DType t = sizeof(T) == 4 ? DType::F32 : DType::F64;
        MX_CUDA(cudaEventRecord(X.ev_fork, st));
        if constexpr (sizeof(T) == 4) spmv_f32(L, x, yfp, nullptr, nullptr, nullptr, st, 0, L.n_first);
        else spmv_f64(L, x, yfp, nullptr, nullptr, nullptr, false, st, 0, L.n_first);
        MX_CUDA(cudaStreamWaitEvent(X.side, X.ev_fork, 0));
        if constexpr (sizeof(T) == 4) spmv_f32(L, x, yfp, nullptr, nullptr, nullptr, X.side, L.n_first, L.nparts);
        else spmv_f64(L, x, yfp, nullptr, nullptr, nullptr, false, X.side, L.n_first, L.nparts);
        MX_CUDA(cudaEventRecord(X.ev_join, X.side));
        const RemoteCounts rcnt(X, P.rank);  // the self slice is read in place after the join
        P.comm->alltoallv(yfp, rcnt.sc.data(), X.sdispl.data(), rb, rcnt.rc.data(), X.rdispl.data(), t, st);  // C
        MX_CUDA(cudaStreamWaitEvent(st, X.ev_join, 0));
        launch_reduce_dot<T>(P, rb, true, y, dot_out, PeerArgs{}, st, yfp + X.sdispl[P.rank]);  // R
        return;
    }
    spmv_any(P, P.fwd, x, yfp, st);                                         // A_p
    exchange_fwd<T>(P, yfp, X.recv_buf.as<T>(), y, st, dot_out);            // R C
}

template <class T>
static void back_t(Plan& P, const T* y, T* x, double* dot_out, cudaStream_t st, bool prepacked = false) {
    if (!P.dist) {
        spmv_any(P, P.back, y, x, st);
        return;
    }
    Exchange& X = P.ex;
    T* yfp = X.y_fp.as<T>();
    exchange_back<T>(P, y, X.recv_buf.as<T>(), yfp, st, prepacked);         // C^T R^T
    double* part = dot_out ? X.dot_part.p() : nullptr;                      // A_p^T
    if constexpr (sizeof(T) == 4) spmv_f32(P.back, yfp, x, part, dot_out, X.tickets.p() + 4, st);
    else spmv_f64(P.back, yfp, x, part, dot_out, X.tickets.p() + 4, false, st);
}

// ---- K slices at once (slice-major vectors): one matrix stream per group of <= 8 slices -----
namespace {

// largest power of two <= min(remaining, what the stage buffer admits)
int group_size(const Plan& P, int remaining) {
    const int kmax = std::min(spmm_max_slices(P.fwd), spmm_max_slices(P.back));
    int k = 1;
    while (k * 2 <= std::min(remaining, kmax)) k *= 2;
    return k;
}

// Sized for the largest group (not the call's), so a buffer allocated here never moves under a
// graph captured by an earlier call with fewer slices.
void ensure_batch_scratch(Plan& P) {
    const int kmax = group_size(P, 8);
    if (kmax <= 1) return;
    const int64_t ncols = std::max({P.fwd.ncols, P.back.ncols, (int64_t)1});
    const size_t xi_bytes = sizeof(float) * (size_t)ncols * kmax;
    grow(P.retired, P.spmm_xi, xi_bytes);
    Exchange& X = P.ex;
    if (P.dist && X.batch_cap < kmax) {
        grow(P.retired, X.y_fp_b, sizeof(float) * std::max<int64_t>(P.nfp, 1) * kmax);
        grow(P.retired, X.recv_b, sizeof(float) * std::max<int64_t>(X.nrecv, 1) * kmax);
        X.batch_cap = kmax;
    }
}

}  // namespace

// Grow-only (common.h: grow), so solves captured against earlier buffers stay valid and nothing
// is freed (no device-wide synchronisation while virtual ranks' peer kernels spin).  No-op under
// capture: cg_run calls this before it captures.
void prepare_batch_scratch(Plan& P, cudaStream_t st) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    MX_CUDA(cudaStreamIsCapturing(st, &cs));
    if (cs != cudaStreamCaptureStatusNone) return;  // under capture: cg_run allocated them already
    const int kmax = group_size(P, 8);
    const int64_t ncols = std::max({P.fwd.ncols, P.back.ncols, (int64_t)1});
    if (kmax <= 1 || (P.spmm_xi.bytes() >= sizeof(float) * (size_t)ncols * kmax &&
                      (!P.dist || P.ex.batch_cap >= kmax)))
        return;
    ensure_batch_scratch(P);
}

void apply_forward_batch(Plan& P, int K, const float* x, float* y, cudaStream_t st) {
    const int64_t nx = P.local_len(0), ny = P.local_len(1);
    prepare_batch_scratch(P, st);
    float* xi = P.spmm_xi.as<float>();
    for (int s0 = 0; s0 < K;) {
        const int k = group_size(P, K - s0);
        const float* xs = x + s0 * nx;
        float* ys = y + s0 * ny;
        if (!P.dist) {
            spmm_f32(P.fwd, k, xs, nx, ys, ny, xi, st);
        } else {
            Exchange& X = P.ex;
            float* yfp = X.y_fp_b.as<float>();
            float* rb = X.recv_b.as<float>();
            spmm_f32(P.fwd, k, xs, nx, yfp, P.nfp, xi, st);                       // A_p, k slices
            for (int s = 0; s < k; ++s)
                exchange_fwd<float>(P, yfp + s * P.nfp, rb + s * X.nrecv, ys + s * ny, st);  // R C
        }
        s0 += k;
    }
}

void apply_back_batch(Plan& P, int K, const float* y, float* x, cudaStream_t st) {
    const int64_t nx = P.local_len(0), ny = P.local_len(1);
    prepare_batch_scratch(P, st);
    float* xi = P.spmm_xi.as<float>();
    for (int s0 = 0; s0 < K;) {
        const int k = group_size(P, K - s0);
        const float* ys = y + s0 * ny;
        float* xs = x + s0 * nx;
        if (!P.dist) {
            spmm_f32(P.back, k, ys, ny, xs, nx, xi, st);
        } else {
            Exchange& X = P.ex;
            float* yfp = X.y_fp_b.as<float>();
            float* rb = X.recv_b.as<float>();
            for (int s = 0; s < k; ++s)
                exchange_back<float>(P, ys + s * ny, rb + s * X.nrecv, yfp + s * P.nfp, st);  // C^T R^T
            spmm_f32(P.back, k, yfp, P.nfp, xs, nx, xi, st);                      // A_p^T, k slices
        }
        s0 += k;
    }
}

// Device time of the communication steps alone (C + R forward, R^T + C^T back), averaged over
// `reps` back-to-back repetitions with CUDA events on `st` -- the "exchange time per iteration"
// of the north star (one forward + one back exchange per CG iteration).
void time_exchange(Plan& P, int reps, double* us_fwd, double* us_back, cudaStream_t st) {
    *us_fwd = *us_back = 0.0;
    if (!P.dist || reps < 1) return;
    Exchange& X = P.ex;
    const int64_t nown = P.s1 - P.s0;
    DevBuf own(P.esize * std::max<int64_t>(nown, 1));
    MX_CUDA(cudaMemsetAsync(own.get(), 0, P.esize * std::max<int64_t>(nown, 1), st));
    MX_CUDA(cudaMemsetAsync(X.y_fp.get(), 0, P.esize * std::max<int64_t>(P.nfp, 1), st));
    cudaEvent_t e[3];
    for (auto& ev : e) MX_CUDA(cudaEventCreate(&ev));
    auto fwd = [&] {
        if (P.esize == 4) exchange_fwd<float>(P, X.y_fp.as<float>(), X.recv_buf.as<float>(), own.as<float>(), st);
        else exchange_fwd<double>(P, X.y_fp.as<double>(), X.recv_buf.as<double>(), own.as<double>(), st);
    };
    auto back = [&] {
        if (P.esize == 4) exchange_back<float>(P, own.as<float>(), X.recv_buf.as<float>(), X.y_fp.as<float>(), st);
        else exchange_back<double>(P, own.as<double>(), X.recv_buf.as<double>(), X.y_fp.as<double>(), st);
    };
    fwd();
    back();  // warm-up
    MX_CUDA(cudaEventRecord(e[0], st));
    for (int i = 0; i < reps; ++i) fwd();
    MX_CUDA(cudaEventRecord(e[1], st));
    for (int i = 0; i < reps; ++i) back();
    MX_CUDA(cudaEventRecord(e[2], st));
    MX_CUDA(cudaEventSynchronize(e[2]));
    float a = 0.f, b = 0.f;
    MX_CUDA(cudaEventElapsedTime(&a, e[0], e[1]));
    MX_CUDA(cudaEventElapsedTime(&b, e[1], e[2]));
    for (auto& ev : e) cudaEventDestroy(ev);
    *us_fwd = 1e3 * a / reps;
    *us_back = 1e3 * b / reps;
}

// Local (non-collective) device time of the A_p and A_p^T kernels alone -- the compute share of
// an iteration, next to time_exchange's communication share.  Zero inputs (the access pattern
// does not depend on values), `reps` back-to-back launches per direction, CUDA events on `st`.
void time_spmv(Plan& P, int reps, double* us_fwd, double* us_back, cudaStream_t st) {
    *us_fwd = *us_back = 0.0;
    if (reps < 1) return;
    const int64_t ntomo = std::max<int64_t>(P.t1 - P.t0, 1);
    const int64_t nsino = std::max<int64_t>(P.dist ? P.nfp : P.s1 - P.s0, 1);
    DevBuf xt(P.esize * ntomo), ys(P.esize * nsino);
    MX_CUDA(cudaMemsetAsync(xt.get(), 0, P.esize * ntomo, st));
    MX_CUDA(cudaMemsetAsync(ys.get(), 0, P.esize * nsino, st));
    auto run = [&](bool fwd) {
        const Layout& L = fwd ? P.fwd : P.back;
        void* in = fwd ? xt.get() : ys.get();
        void* out = fwd ? ys.get() : xt.get();
        if (P.esize == 4) spmv_any(P, L, static_cast<const float*>(in), static_cast<float*>(out), st);
        else spmv_any(P, L, static_cast<const double*>(in), static_cast<double*>(out), st);
    };
    run(true);
    run(false);  // warm-up
    cudaEvent_t e[3];
    for (auto& ev : e) MX_CUDA(cudaEventCreate(&ev));
    MX_CUDA(cudaEventRecord(e[0], st));
    for (int i = 0; i < reps; ++i) run(true);
    MX_CUDA(cudaEventRecord(e[1], st));
    for (int i = 0; i < reps; ++i) run(false);
    MX_CUDA(cudaEventRecord(e[2], st));
    MX_CUDA(cudaEventSynchronize(e[2]));
    float a = 0.f, b = 0.f;
    MX_CUDA(cudaEventElapsedTime(&a, e[0], e[1]));
    MX_CUDA(cudaEventElapsedTime(&b, e[1], e[2]));
    for (auto& ev : e) cudaEventDestroy(ev);
    *us_fwd = 1e3 * a / reps;
    *us_back = 1e3 * b / reps;
}

void preload_exchange_kernels() {
    cudaFuncAttributes fa;
    MX_CUDA(cudaFuncGetAttributes(&fa, reduce_dot_kernel<float>));
    MX_CUDA(cudaFuncGetAttributes(&fa, reduce_dot_kernel<double>));
    MX_CUDA(cudaFuncGetAttributes(&fa, pack_kernel<float>));
    MX_CUDA(cudaFuncGetAttributes(&fa, pack_self_kernel<float>));
}

void reduce_partials(Plan& P, const float* recv, float* y, double* dot_out, const PeerArgs& pa, cudaStream_t st) {
    launch_reduce_dot<float>(P, recv, true, y, dot_out, pa, st);
}

void apply_forward(Plan& P, const void* x, void* y, cudaStream_t st, double* dot_out) {
    if (P.ex.peer) peer_forward(P, (const float*)x, (float*)y, dot_out, st);
    else if (P.esize == 4) forward_t<float>(P, (const float*)x, (float*)y, dot_out, st);
    else forward_t<double>(P, (const double*)x, (double*)y, dot_out, st);
}

void apply_back(Plan& P, const void* y, void* x, cudaStream_t st, double* dot_out, bool prepacked) {
    if (P.ex.peer) peer_back(P, (const float*)y, (float*)x, dot_out, st);
    else if (P.esize == 4) back_t<float>(P, (const float*)y, (float*)x, dot_out, st, prepacked);
    else back_t<double>(P, (const double*)y, (double*)x, dot_out, st, prepacked);
}

bool cg_fused_pack(const Plan& P) {
    static const bool on = [] {
        const char* e = std::getenv("MEMXCT_CG_FUSED_PACK");
        return !(e && e[0] == '0');
    }();
    return on && P.dist && !P.shard && !P.ex.peer && !P.ex.dense && P.ex.nrecv > 0;
}

PackTargets pack_targets(Plan& P) {
    Exchange& X = P.ex;
    PackTargets t;
    t.red_ptr = X.red_ptr.p();
    t.red_pos = X.red_pos.p();
    t.rb = X.recv_buf.get();
    t.self = static_cast<char*>(X.y_fp.get()) + P.esize * X.sdispl[P.rank];
    t.lo = X.rdispl[P.rank];
    t.hi = X.rdispl[P.rank + 1];
    return t;
}

}  // namespace mx
