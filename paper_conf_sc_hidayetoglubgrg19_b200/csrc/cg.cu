// cg.cu -- CGLS driver (sec. 3.5.2; readings R13-R16), for one slice or a batch of K
// slices that share the memoized matrices.
//
// Recursive-residual CGLS per slice, x0 = 0 (reading R14), exactly `iters` iterations:
//   setup:  r = y;  s = A^T r;  p = s;  gamma_0 = <s,s>;  res_0 = ||r||
//   iter k: q = A p, delta_k = <q,q>
//           alpha = gamma_{k-1} / delta_k;  x = fma(alpha, p, x);  r = fma(-alpha, q, r)
//           s = A^T r, gamma_k = <s,s>
//           beta = gamma_k / gamma_{k-1};  p = fma(beta, p, s)
// CG_VARIANT = 1 recomputes the residual explicitly, r = y - A x (2 forward + 1 back).
// Vectors of a batch are slice-major ([K][n]); every vector kernel runs a grid of
// (blocks, K) with slice = blockIdx.y, and the per-slice arithmetic (including the reduction
// order of the dots) is exactly the single-slice one, so slice s of a batch reproduces a
// single-slice solve bit for bit.  Scalars live on the device (one slot per slice and
// iteration), so the whole solve is one CUDA graph.  Iterations after gamma or delta reach 0 are
// no-ops, like the oracle's early exit.
#include "plan.h"

namespace mx {

namespace {

constexpr int kVT = 256;
// Vector steps are HBM streams of a few MB: 8 CTAs x 256 threads per SM and 4 independent
// elements per thread per pass keep ~10 MB of loads in flight (296 CTAs with one element per
// pass ran at ~1 TB/s: 32 us for the 30 MB of the x/r update at cfg3).
constexpr int kVecCtasPerSm = 8;
constexpr int kU = 4;
int vec_blocks_max() { return kVecCtasPerSm * num_sms(); }

// scalar slots of slice s: gam[s*n1 + k], del[...], res2[...]; stop flags per slice
struct Scal {
    double* gam;
    double* del;
    double* res2;
    int* stop;     // [K]  iterations stopped (gamma or delta reached 0)
    int* stop_at;  // [K]  first iteration that did not run
    int32_t n1;    // iters + 1
};

int64_t scal_doubles(int32_t iters, int32_t K) { return 3 * (int64_t)(iters + 1) * K + K; }

Scal scal_of(Plan& P) {
    const int32_t n1 = (int32_t)P.scal_iters + 1, K = P.scal_slices;
    Scal s;
    s.n1 = n1;
    s.gam = P.scal.p();
    s.del = s.gam + (int64_t)n1 * K;
    s.res2 = s.del + (int64_t)n1 * K;
    s.stop = reinterpret_cast<int*>(s.res2 + (int64_t)n1 * K);
    s.stop_at = s.stop + K;
    return s;
}

// block-wide deterministic reduction + last-block finish (fixed order); per slice blockIdx.y
__device__ void vec_dot_finish(double mine, double* part, double* out, unsigned int* ticket) {
    __shared__ double red[kVT / 32];
    __shared__ bool am_last;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    part += (int64_t)blockIdx.y * gridDim.x;
    ticket += blockIdx.y;
    for (int o = 16; o; o >>= 1) mine += __shfl_xor_sync(0xffffffffu, mine, o);
    if (lane == 0) red[warp] = mine;
    __syncthreads();
    if (threadIdx.x == 0) {
        double s = 0.0;
        for (int w = 0; w < kVT / 32; ++w) s += red[w];
        part[blockIdx.x] = s;
        __threadfence();
        am_last = (atomicAdd(ticket, 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (!am_last) return;
    __threadfence();
    // fixed-order parallel sum of the per-block partials: thread t adds blocks t, t + kVT, ...
    double t = 0.0;
    for (unsigned i = threadIdx.x; i < gridDim.x; i += kVT) t += ((volatile double*)part)[i];
    for (int o = 16; o; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
    __syncthreads();
    if (lane == 0) red[warp] = t;
    __syncthreads();
    if (threadIdx.x == 0) {
        double tot = 0.0;
        for (int w = 0; w < kVT / 32; ++w) tot += red[w];
        *out = tot;
        *ticket = 0u;
    }
}

#define MX_GRID_LOOP(i, n) for (int64_t i = (int64_t)blockIdx.x * kVT + threadIdx.x; i < (n); i += (int64_t)gridDim.x * kVT)
// kU elements per thread per pass, strided by the grid so every warp access stays coalesced:
// body(i) for i = i0 + u * stride, u < kU, i < n (loads of the kU elements are independent)
#define MX_GRID_LOOP_U(i, n, body)                                                                \
    for (int64_t i##0 = (int64_t)blockIdx.x * kVT + threadIdx.x, i##s = (int64_t)gridDim.x * kVT; \
         i##0 < (n); i##0 += kU * i##s) {                                                          \
        _Pragma("unroll") for (int u_ = 0; u_ < kU; ++u_) {                                        \
            const int64_t i = i##0 + u_ * i##s;                                                    \
            if (i < (n)) { body }                                                                  \
        }                                                                                          \
    }

// r = y ; x = 0 ; res2[0] = <r, r> ; stop = 0
template <class T>
__global__ void __launch_bounds__(kVT)
cg_init_kernel(const T* __restrict__ y, T* __restrict__ r, int64_t nr, T* __restrict__ x, int64_t nx,
               Scal sc, double* part, unsigned int* ticket) {
    const int s = blockIdx.y;
    y += s * nr; r += s * nr; x += s * nx;
    double acc = 0.0;
    MX_GRID_LOOP_U(i, nr, const T v = y[i]; r[i] = v; acc += (double)v * (double)v;)
    MX_GRID_LOOP_U(i, nx, x[i] = T(0);)
    if (blockIdx.x == 0 && threadIdx.x == 0) { sc.stop[s] = 0; sc.stop_at[s] = 0x7fffffff; }
    vec_dot_finish(acc, part, sc.res2 + (int64_t)s * sc.n1, ticket);
}

template <class T>
__global__ void __launch_bounds__(kVT) copy_kernel(const T* __restrict__ a, T* __restrict__ b, int64_t n) {
    a += blockIdx.y * n; b += blockIdx.y * n;
    MX_GRID_LOOP_U(i, n, b[i] = a[i];)
}

__device__ __forceinline__ float upd(float a, double s, float b) { return (float)__fma_rn(s, (double)a, (double)b); }
__device__ __forceinline__ double upd(double a, double s, double b) { return __fma_rn(s, a, b); }

// alpha = gam[k-1] / del[k]; x = fma(alpha, p, x); r = fma(-alpha, q, r); res2[k] = <r, r>
// kPack (P > 1, sparse collective exchange): also the R^T pack of the next back projection --
// the new r[i] goes to every pack position of owned ray i (pk.red_pos[pk.red_ptr[i] ..]), its own
// slice in place in the footprint buffer.  Same grid and element map, so the dot is unchanged.
template <class T, bool kUpdateR, bool kPack = false>
__global__ void __launch_bounds__(kVT)
cg_update_xr_kernel(T* __restrict__ x, const T* __restrict__ p, int64_t nx, T* __restrict__ r,
                    const T* __restrict__ q, int64_t nr, Scal sc, int32_t k, double* part,
                    unsigned int* ticket, PackTargets pk = PackTargets{}) {
    const int s = blockIdx.y;
    const int64_t o = (int64_t)s * sc.n1;
    x += s * nx; p += s * nx; r += s * nr; q += s * nr;
    const double g = sc.gam[o + k - 1], d = sc.del[o + k];
    if (sc.stop[s] || g == 0.0 || d == 0.0) {
        if (blockIdx.x == 0 && threadIdx.x == 0 && !sc.stop[s]) { sc.stop[s] = 1; sc.stop_at[s] = k; }
        return;
    }
    const double alpha = __ddiv_rn(g, d);
    MX_GRID_LOOP_U(i, nx, x[i] = upd(p[i], alpha, x[i]);)
    if (kUpdateR) {
        double acc = 0.0;
        if constexpr (kPack) {
            T* rb = static_cast<T*>(pk.rb);
            T* self = static_cast<T*>(pk.self);
            MX_GRID_LOOP_U(i, nr, const T v = upd(q[i], -alpha, r[i]); r[i] = v; acc += (double)v * (double)v;
                           for (int64_t e = pk.red_ptr[i]; e < pk.red_ptr[i + 1]; ++e) {
                               const int64_t j = pk.red_pos[e];
                               if (j >= pk.lo && j < pk.hi) self[j - pk.lo] = v; else rb[j] = v;
                           })
        } else {
            MX_GRID_LOOP_U(i, nr, const T v = upd(q[i], -alpha, r[i]); r[i] = v; acc += (double)v * (double)v;)
        }
        vec_dot_finish(acc, part, sc.res2 + o + k, ticket);
    }
}

// explicit residual (CG_VARIANT 1): r = y - ax ; res2[k] = <r, r>
template <class T>
__global__ void __launch_bounds__(kVT)
cg_explicit_r_kernel(const T* __restrict__ y, const T* __restrict__ ax, T* __restrict__ r, int64_t nr,
                     Scal sc, int32_t k, double* part, unsigned int* ticket) {
    const int s = blockIdx.y;
    if (sc.stop[s]) return;
    y += s * nr; ax += s * nr; r += s * nr;
    double acc = 0.0;
    MX_GRID_LOOP_U(i, nr, const T v = y[i] - ax[i]; r[i] = v; acc += (double)v * (double)v;)
    vec_dot_finish(acc, part, sc.res2 + (int64_t)s * sc.n1 + k, ticket);
}

// beta = gam[k] / gam[k-1]; p = fma(beta, p, s)
template <class T>
__global__ void __launch_bounds__(kVT)
cg_update_p_kernel(T* __restrict__ p, const T* __restrict__ sv, int64_t nx, Scal sc, int32_t k) {
    const int s = blockIdx.y;
    if (sc.stop[s]) return;
    const int64_t o = (int64_t)s * sc.n1;
    p += s * nx; sv += s * nx;
    const double beta = __ddiv_rn(sc.gam[o + k], sc.gam[o + k - 1]);
    MX_GRID_LOOP_U(i, nx, p[i] = upd(p[i], beta, sv[i]);)
}

// <v, v> in fp64 over a fixed grid (deterministic: fixed element->thread map, fixed tree);
// out[s * stride] for slice s = blockIdx.y
template <class T>
__global__ void __launch_bounds__(kVT)
dot_kernel(const T* __restrict__ v, int64_t n, double* out, int64_t stride, double* part, unsigned int* ticket) {
    v += blockIdx.y * n;
    double acc = 0.0;
    MX_GRID_LOOP_U(i, n, const double e = (double)v[i]; acc += e * e;)
    vec_dot_finish(acc, part, out + blockIdx.y * stride, ticket);
}

unsigned vec_blocks(int64_t n) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(vec_blocks_max(), ceil_div(n, (int64_t)kVT * kU)));
}

// CG dots at P > 1: one fp64 per slice summed over the ranks -- over peer memory with the fused
// exchange (peer_allreduce, rank order), else by the transport's allreduce (NCCL / virtual ranks).
void allreduce_slices(Plan& P, double* v, int K, int64_t stride, cudaStream_t st, bool in_kernel = false) {
    if (!P.dist || in_kernel) return;
    if (P.ex.peer) {
        peer_allreduce(P, v, K, stride, st);
        return;
    }
    for (int s = 0; s < K; ++s) P.comm->allreduce_sum(v + s * stride, 1, DType::F64, st);
}

// Projection of K slices followed by the per-slice dot of the output.  At K = 1, P = 1 the dot
// is fused into the SpMV epilogue: canonical mode as per-partition fma chains (reading R16),
// otherwise as a per-CTA tree + last-CTA sum in partition order (deterministic).  (With the
// first, uniform-width kernel that epilogue cost 0.5 ms per 2 ms SpMV, profiles/r01a_launches.md;
// with the jagged kernel it is free, so it is the default; MEMXCT_FUSED_DOT=0 selects the
// separate dot kernel.)  P > 1 (the projection includes the exchange, A = R C A_p): the local
// dot is fused into the last kernel of the projection -- the reduction R forward, A_p^T back --
// and summed over the ranks.  Batched: separate dot kernels.
template <class T>
void op_dir(Plan& P, bool forward, int K, const T* in, T* out, double* dot_out, int64_t dot_stride,
            cudaStream_t st, bool prepacked = false) {
    // P > 1: the rank's local dot is fused into the reduction R (forward) or into A_p^T's
    // epilogue (back) for every exchange, then summed over the ranks (allreduce_slices)
    const bool fused = dot_out && K == 1 && (P.dist || P.opt.canonical != 0 || P.fused_dot);
    if (!P.dist && K == 1) {
        const Layout& L = forward ? P.fwd : P.back;
        double* part = forward ? P.part_fwd.p() : P.part_back.p();
        if constexpr (sizeof(T) == 4)
            spmv_f32(L, in, out, part, fused ? dot_out : nullptr, P.tickets.p(), st);
        else
            spmv_f64(L, in, out, part, fused ? dot_out : nullptr, P.tickets.p(), P.opt.canonical != 0, st);
    } else if (K == 1) {
        if (forward) apply_forward(P, in, out, st, fused ? dot_out : nullptr);
        else apply_back(P, in, out, st, fused ? dot_out : nullptr, prepacked);
    } else {
        if constexpr (sizeof(T) == 4) {
            if (forward) apply_forward_batch(P, K, in, out, st);
            else apply_back_batch(P, K, in, out, st);
        } else {
            fail(MEMXCT_ERR_UNSUPPORTED, "multi-slice CG is FP32 only");
        }
    }
    if (dot_out && !fused) {
        const int64_t n = P.local_len(forward ? 1 : 0);
        dot_kernel<T><<<dim3(vec_blocks(n), K), kVT, 0, st>>>(out, n, dot_out, dot_stride, P.part_vec.p(),
                                                              P.tickets.p() + 64);
        MX_LAUNCHED();
    }
    // fused peer exchange with folded waits: the last kernel of the projection already summed
    // the dot over the ranks (peer_dot_allreduce)
    const bool summed = fused && P.ex.peer && P.ex.fold;
    if (dot_out && P.dist) allreduce_slices(P, dot_out, K, dot_stride, st, summed);
}

template <class T>
void cg_enqueue(Plan& P, const T* y, T* x, int32_t iters, int K, cudaStream_t st) {
    const int64_t nx = P.local_len(0), nr = P.local_len(1);
    T* r = P.cg_r.as<T>();
    T* q = P.cg_q.as<T>();
    T* s = P.cg_s.as<T>();
    T* p = P.cg_p.as<T>();
    T* ax = P.cg_ax.as<T>();
    const Scal sc = scal_of(P);
    double* vpart = P.part_vec.p();
    unsigned int* tick = P.tickets.p() + 32;
    const unsigned gb = vec_blocks(std::max(nx, nr));
    // sparse collective exchange, one slice: the back projection's R^T pack rides on the r update
    const bool packed = K == 1 && P.opt.cg_variant == 0 && cg_fused_pack(P);
    cg_init_kernel<T><<<dim3(gb, K), kVT, 0, st>>>(y, r, nr, x, nx, sc, vpart, tick);
    MX_LAUNCHED();
    op_dir<T>(P, false, K, r, s, sc.gam, sc.n1, st);                    // s = A^T r, gamma_0
    copy_kernel<T><<<dim3(vec_blocks(nx), K), kVT, 0, st>>>(s, p, nx);  // p = s
    MX_LAUNCHED();
    for (int32_t k = 1; k <= iters; ++k) {
        op_dir<T>(P, true, K, p, q, sc.del + k, sc.n1, st);             // q = A p, delta_k
        if (P.opt.cg_variant == 1) {
            cg_update_xr_kernel<T, false><<<dim3(vec_blocks(nx), K), kVT, 0, st>>>(x, p, nx, r, q, nr, sc, k,
                                                                                    vpart, tick);
            MX_LAUNCHED();
            op_dir<T>(P, true, K, x, ax, nullptr, 0, st);                // ax = A x
            cg_explicit_r_kernel<T><<<dim3(vec_blocks(nr), K), kVT, 0, st>>>(y, ax, r, nr, sc, k, vpart, tick);
            MX_LAUNCHED();
        } else if (packed) {  // + the R^T pack of the back projection below
            cg_update_xr_kernel<T, true, true><<<dim3(gb, K), kVT, 0, st>>>(x, p, nx, r, q, nr, sc, k, vpart, tick,
                                                                            pack_targets(P));
            MX_LAUNCHED();
        } else {
            cg_update_xr_kernel<T, true><<<dim3(gb, K), kVT, 0, st>>>(x, p, nx, r, q, nr, sc, k, vpart, tick);
            MX_LAUNCHED();
        }
        op_dir<T>(P, false, K, r, s, sc.gam + k, sc.n1, st, packed);    // s = A^T r, gamma_k
        cg_update_p_kernel<T><<<dim3(vec_blocks(nx), K), kVT, 0, st>>>(p, s, nx, sc, k);
        MX_LAUNCHED();
    }
    // ||r_k||^2 only reports (no step depends on it): the local partials of every iteration are
    // summed over the ranks once, after the loop -- one collective per slice per solve instead of
    // one per iteration.  Iterations that did not run are ignored by cg_fetch_norms.
    if (P.dist)
        for (int sl = 0; sl < K; ++sl) P.comm->allreduce_sum(sc.res2 + (int64_t)sl * sc.n1, iters + 1, DType::F64, st);
}

void cg_enqueue_any(Plan& P, const void* y, void* x, int32_t iters, int K, cudaStream_t st) {
    if (P.esize == 4) cg_enqueue<float>(P, (const float*)y, (float*)x, iters, K, st);
    else cg_enqueue<double>(P, (const double*)y, (double*)x, iters, K, st);
}

}  // namespace

void cg_run(Plan& P, const void* y, void* x, int32_t iters, int32_t K, cudaStream_t st) {
    if (K < 1 || K > 64) fail(MEMXCT_ERR_INVALID_ARG, "slices must be in [1, 64]");
    if (K > 1 && P.esize != 4) fail(MEMXCT_ERR_UNSUPPORTED, "multi-slice CG is FP32 only");
    const int64_t nx = P.local_len(0), nr = P.local_len(1);
    // grow-only (common.h: grow): no cudaFree while peers' kernels may wait on this rank
    if (K > P.cg_slices) {
        MX_CUDA(cudaStreamSynchronize(st));
        grow(P.retired, P.cg_r, P.esize * std::max<int64_t>(nr, 1) * K);
        grow(P.retired, P.cg_q, P.esize * std::max<int64_t>(nr, 1) * K);
        grow(P.retired, P.cg_s, P.esize * std::max<int64_t>(nx, 1) * K);
        grow(P.retired, P.cg_p, P.esize * std::max<int64_t>(nx, 1) * K);
        if (P.opt.cg_variant == 1) grow(P.retired, P.cg_ax, P.esize * std::max<int64_t>(nr, 1) * K);
        grow(P.retired, P.part_fwd, std::max<int64_t>(P.fwd.nparts, 1));
        grow(P.retired, P.part_back, std::max<int64_t>(P.back.nparts, 1));
        grow(P.retired, P.part_vec, (int64_t)vec_blocks_max() * K);
        if (!P.tickets.p()) {
            P.tickets.alloc(128);
            MX_CUDA(cudaMemsetAsync(P.tickets.p(), 0, 128 * sizeof(unsigned int), st));
        }
        P.cg_slices = K;
        P.graphs.clear();  // captured against the previous buffers (still allocated)
    }
    if (iters > P.scal_iters || K > P.scal_slices) {
        MX_CUDA(cudaStreamSynchronize(st));
        P.graphs.clear();  // the scalar layout (stride iters + 1) changes
        P.scal_iters = std::max<int64_t>(iters, P.scal_iters);
        P.scal_slices = std::max<int32_t>(K, P.scal_slices);
        const int64_t nd = scal_doubles((int32_t)P.scal_iters, P.scal_slices);
        grow(P.retired, P.scal, nd);
        MX_CUDA(cudaMemsetAsync(P.scal.p(), 0, 8 * nd, st));
    }
    if (K > 1) prepare_batch_scratch(P, st);
    if (P.dist && !P.comm->capturable()) {  // virtual ranks: eager launches
        cg_enqueue_any(P, y, x, iters, K, st);
        return;
    }
    auto key = std::make_tuple(y, x, iters * 64 + K, st);
    auto it = P.graphs.find(key);
    if (it == P.graphs.end()) {
        if (P.graphs.size() >= kMaxGraphs) {  // evict the least recently used solve
            auto lru = P.graphs.begin();
            for (auto g = P.graphs.begin(); g != P.graphs.end(); ++g)
                if (g->second->last_used < lru->second->last_used) lru = g;
            MX_CUDA(cudaStreamSynchronize(st));
            P.graphs.erase(lru);
        }
        // capture the whole solve once on a private stream, replay it on the caller's stream
        MX_CUDA(cudaStreamSynchronize(st));
        cudaStream_t cap;
        MX_CUDA(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
        cudaGraph_t g = nullptr;
        MX_CUDA(cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal));
        const int64_t before = launch_count();
        try {
            cg_enqueue_any(P, y, x, iters, K, cap);
        } catch (...) {
            cudaStreamEndCapture(cap, &g);
            if (g) cudaGraphDestroy(g);
            cudaStreamDestroy(cap);
            throw;
        }
        const int64_t captured = launch_count() - before;
        count_launch(-captured);  // captured, not launched: counted at every graph launch
        MX_CUDA(cudaStreamEndCapture(cap, &g));
        auto cgg = std::make_unique<CgGraph>();
        cgg->nkernels = captured;
        cudaError_t e = cudaGraphInstantiate(&cgg->exec, g, 0);
        cudaGraphDestroy(g);
        cudaStreamDestroy(cap);
        MX_CUDA(e);
        it = P.graphs.emplace(key, std::move(cgg)).first;
    }
    it->second->last_used = ++P.graph_clock;
    MX_CUDA(cudaGraphLaunch(it->second->exec, st));
    count_launch(it->second->nkernels);
    MX_CUDA(cudaGetLastError());
}

void cg_fetch_norms(Plan& P, int32_t iters, int32_t K, double* out, cudaStream_t st) {
    const Scal sc = scal_of(P);
    std::vector<double> res2((size_t)sc.n1 * K);
    std::vector<int> stop_at(K);
    MX_CUDA(cudaMemcpyAsync(res2.data(), sc.res2, 8 * (size_t)sc.n1 * K, cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaMemcpyAsync(stop_at.data(), sc.stop_at, sizeof(int) * K, cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    for (int s = 0; s < K; ++s) {
        double* o = out + (int64_t)s * (iters + 1);
        for (int32_t k = 0; k <= iters; ++k) {
            if (k >= stop_at[s]) o[k] = o[k - 1];  // iterations that did not run repeat the last norm
            else o[k] = std::sqrt(res2[(size_t)s * sc.n1 + k]);
        }
    }
}

}  // namespace mx
