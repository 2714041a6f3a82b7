// cg.cu -- CGLS driver (sec. 3.5.2; readings R13-R16).
//
// Recursive-residual CGLS, x0 = 0 (reading R14), exactly `iters` iterations:
//   setup:  r = y;  s = A^T r;  p = s;  gamma_0 = <s,s>;  res_0 = ||r||
//   iter k: q = A p, delta_k = <q,q>          (dot fused into the forward SpMV epilogue)
//           alpha = gamma_{k-1} / delta_k;  x = fma(alpha, p, x);  r = fma(-alpha, q, r)
//           s = A^T r, gamma_k = <s,s>        (dot fused into the back SpMV epilogue)
//           beta = gamma_k / gamma_{k-1};  p = fma(beta, p, s)
// CG_VARIANT = 1 recomputes the residual explicitly, r = y - A x (2 forward + 1 back).
// Scalars live on the device (one slot per iteration), so the whole solve is one CUDA graph:
// no host round trip per iteration.  Iterations after gamma or delta reach 0 are no-ops, like
// the oracle's early exit.
#include "plan.h"

namespace mx {

namespace {

constexpr int kVT = 256;
constexpr int kVecBlocks = 296;  // 2 x 148 SMs

// scalar slots
struct Scal {
    double* gam;   // [iters + 1]
    double* del;   // [iters + 1]
    double* res2;  // [iters + 1]
    int* stop;     // [1]  iterations stopped (gamma or delta reached 0)
    int* stop_at;  // [1]  first iteration that did not run
};

Scal scal_of(Plan& P, int32_t iters) {
    Scal s;
    s.gam = P.scal.p();
    s.del = s.gam + (iters + 1);
    s.res2 = s.del + (iters + 1);
    s.stop = reinterpret_cast<int*>(s.res2 + (iters + 1));
    s.stop_at = s.stop + 1;
    return s;
}

// block-wide deterministic reduction + last-block finish (fixed order)
__device__ void vec_dot_finish(double mine, double* part, double* out, unsigned int* ticket) {
    __shared__ double red[kVT / 32];
    __shared__ bool am_last;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
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
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (unsigned i = 0; i < gridDim.x; ++i) t += ((volatile double*)part)[i];
        *out = t;
        *ticket = 0u;
    }
}

// r = y ; x = 0 ; res2[0] = <r, r> ; stop = 0
template <class T>
__global__ void __launch_bounds__(kVT)
cg_init_kernel(const T* __restrict__ y, T* __restrict__ r, int64_t nr, T* __restrict__ x, int64_t nx,
               Scal sc, double* part, unsigned int* ticket) {
    double acc = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * kVT + threadIdx.x; i < nr; i += (int64_t)gridDim.x * kVT) {
        const T v = y[i];
        r[i] = v;
        acc += (double)v * (double)v;
    }
    for (int64_t i = (int64_t)blockIdx.x * kVT + threadIdx.x; i < nx; i += (int64_t)gridDim.x * kVT) x[i] = T(0);
    if (blockIdx.x == 0 && threadIdx.x == 0) { *sc.stop = 0; *sc.stop_at = 0x7fffffff; }
    vec_dot_finish(acc, part, sc.res2, ticket);
}

template <class T>
__global__ void copy_kernel(const T* __restrict__ a, T* __restrict__ b, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        b[i] = a[i];
}

__device__ __forceinline__ float upd(float a, double s, float b) { return (float)__fma_rn(s, (double)a, (double)b); }
__device__ __forceinline__ double upd(double a, double s, double b) { return __fma_rn(s, a, b); }

// alpha = gam[k-1] / del[k]; x = fma(alpha, p, x); r = fma(-alpha, q, r); res2[k] = <r, r>
template <class T, bool kUpdateR>
__global__ void __launch_bounds__(kVT)
cg_update_xr_kernel(T* __restrict__ x, const T* __restrict__ p, int64_t nx, T* __restrict__ r,
                    const T* __restrict__ q, int64_t nr, Scal sc, int32_t k, double* part,
                    unsigned int* ticket) {
    const double g = sc.gam[k - 1], d = sc.del[k];
    if (*sc.stop || g == 0.0 || d == 0.0) {
        if (blockIdx.x == 0 && threadIdx.x == 0 && !*sc.stop) { *sc.stop = 1; *sc.stop_at = k; }
        return;
    }
    const double alpha = __ddiv_rn(g, d);
    for (int64_t i = (int64_t)blockIdx.x * kVT + threadIdx.x; i < nx; i += (int64_t)gridDim.x * kVT)
        x[i] = upd(p[i], alpha, x[i]);
    double acc = 0.0;
    if (kUpdateR) {
        for (int64_t i = (int64_t)blockIdx.x * kVT + threadIdx.x; i < nr; i += (int64_t)gridDim.x * kVT) {
            const T v = upd(q[i], -alpha, r[i]);
            r[i] = v;
            acc += (double)v * (double)v;
        }
        vec_dot_finish(acc, part, sc.res2 + k, ticket);
    }
}

// explicit residual (CG_VARIANT 1): r = y - ax ; res2[k] = <r, r>
template <class T>
__global__ void __launch_bounds__(kVT)
cg_explicit_r_kernel(const T* __restrict__ y, const T* __restrict__ ax, T* __restrict__ r, int64_t nr,
                     Scal sc, int32_t k, double* part, unsigned int* ticket) {
    if (*sc.stop) return;
    double acc = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * kVT + threadIdx.x; i < nr; i += (int64_t)gridDim.x * kVT) {
        const T v = y[i] - ax[i];
        r[i] = v;
        acc += (double)v * (double)v;
    }
    vec_dot_finish(acc, part, sc.res2 + k, ticket);
}

// beta = gam[k] / gam[k-1]; p = fma(beta, p, s)
template <class T>
__global__ void __launch_bounds__(kVT)
cg_update_p_kernel(T* __restrict__ p, const T* __restrict__ s, int64_t nx, Scal sc, int32_t k) {
    if (*sc.stop) return;
    const double beta = __ddiv_rn(sc.gam[k], sc.gam[k - 1]);
    for (int64_t i = (int64_t)blockIdx.x * kVT + threadIdx.x; i < nx; i += (int64_t)gridDim.x * kVT)
        p[i] = upd(p[i], beta, s[i]);
}

// <v, v> in fp64 over a fixed grid (deterministic: fixed element->thread map, fixed tree)
template <class T>
__global__ void __launch_bounds__(kVT)
dot_kernel(const T* __restrict__ v, int64_t n, double* out, double* part, unsigned int* ticket) {
    double acc = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * kVT + threadIdx.x; i < n; i += (int64_t)gridDim.x * kVT) {
        const double e = (double)v[i];
        acc += e * e;
    }
    vec_dot_finish(acc, part, out, ticket);
}

unsigned vec_blocks(int64_t n) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(kVecBlocks, ceil_div(n, kVT)));
}

// Projection followed by the dot product of its output.  Canonical mode fuses the dot into the
// SpMV epilogue (per-partition fma chains, reading R16).  Otherwise a separate small dot kernel
// is used: measured on B200, the fused last-CTA epilogue slowed the 2 ms SpMV by ~0.5 ms
// (profiles/r01a_launches.md), while the separate pass over the 4-6 MB vector costs a few us.
// P > 1: the projection includes the exchange (A = R C A_p), and the local dot is allreduced.
template <class T>
void op_dir(Plan& P, bool forward, const T* in, T* out, double* dot_out, cudaStream_t st) {
    const Layout& L = forward ? P.fwd : P.back;
    if (P.nranks == 1) {
        double* part = forward ? P.part_fwd.p() : P.part_back.p();
        const bool fused = dot_out && (P.opt.canonical != 0 || P.fused_dot);
        if constexpr (sizeof(T) == 4)
            spmv_f32(L, in, out, part, fused ? dot_out : nullptr, P.tickets.p(), st);
        else
            spmv_f64(L, in, out, part, fused ? dot_out : nullptr, P.tickets.p(), P.opt.canonical != 0, st);
        if (dot_out && !fused) {
            dot_kernel<T><<<vec_blocks(L.nrows), kVT, 0, st>>>(out, L.nrows, dot_out, P.part_vec.p(),
                                                               P.tickets.p() + 2);
            MX_LAUNCHED();
        }
        return;
    }
    if (forward) apply_forward(P, in, out, st);
    else apply_back(P, in, out, st);
    if (dot_out) {
        const int64_t n = P.local_len(forward ? 1 : 0);
        dot_kernel<T><<<vec_blocks(n), kVT, 0, st>>>(out, n, dot_out, P.part_vec.p(), P.tickets.p() + 2);
        MX_LAUNCHED();
        P.comm->allreduce_sum(dot_out, 1, DType::F64, st);
    }
}

void allreduce_scalar(Plan& P, double* v, cudaStream_t st) {
    if (P.nranks > 1) P.comm->allreduce_sum(v, 1, DType::F64, st);
}

template <class T>
void cg_enqueue(Plan& P, const T* y, T* x, int32_t iters, cudaStream_t st) {
    const int64_t nx = P.local_len(0), nr = P.local_len(1);
    T* r = P.cg_r.as<T>();
    T* q = P.cg_q.as<T>();
    T* s = P.cg_s.as<T>();
    T* p = P.cg_p.as<T>();
    T* ax = P.cg_ax.as<T>();
    const Scal sc = scal_of(P, (int32_t)P.scal_iters);
    double* vpart = P.part_vec.p();
    unsigned int* tick = P.tickets.p() + 1;
    const unsigned gb = vec_blocks(std::max(nx, nr));
    cg_init_kernel<T><<<gb, kVT, 0, st>>>(y, r, nr, x, nx, sc, vpart, tick);
    MX_LAUNCHED();
    allreduce_scalar(P, sc.res2, st);
    op_dir<T>(P, false, r, s, sc.gam, st);                      // s = A^T r, gamma_0
    copy_kernel<T><<<vec_blocks(nx), kVT, 0, st>>>(s, p, nx);  // p = s
    MX_LAUNCHED();
    for (int32_t k = 1; k <= iters; ++k) {
        op_dir<T>(P, true, p, q, sc.del + k, st);               // q = A p, delta_k
        if (P.opt.cg_variant == 1) {
            cg_update_xr_kernel<T, false><<<vec_blocks(nx), kVT, 0, st>>>(x, p, nx, r, q, nr, sc, k, vpart, tick);
            MX_LAUNCHED();
            op_dir<T>(P, true, x, ax, nullptr, st);              // ax = A x
            cg_explicit_r_kernel<T><<<vec_blocks(nr), kVT, 0, st>>>(y, ax, r, nr, sc, k, vpart, tick);
            MX_LAUNCHED();
        } else {
            cg_update_xr_kernel<T, true><<<gb, kVT, 0, st>>>(x, p, nx, r, q, nr, sc, k, vpart, tick);
            MX_LAUNCHED();
        }
        allreduce_scalar(P, sc.res2 + k, st);
        op_dir<T>(P, false, r, s, sc.gam + k, st);              // s = A^T r, gamma_k
        cg_update_p_kernel<T><<<vec_blocks(nx), kVT, 0, st>>>(p, s, nx, sc, k);
        MX_LAUNCHED();
    }
}

void cg_enqueue_any(Plan& P, const void* y, void* x, int32_t iters, cudaStream_t st) {
    if (P.esize == 4) cg_enqueue<float>(P, (const float*)y, (float*)x, iters, st);
    else cg_enqueue<double>(P, (const double*)y, (double*)x, iters, st);
}

}  // namespace

void cg_run(Plan& P, const void* y, void* x, int32_t iters, cudaStream_t st) {
    const int64_t nx = P.local_len(0), nr = P.local_len(1);
    if (!P.cg_r.get()) {
        P.cg_r.alloc(P.esize * std::max<int64_t>(nr, 1));
        P.cg_q.alloc(P.esize * std::max<int64_t>(nr, 1));
        P.cg_s.alloc(P.esize * std::max<int64_t>(nx, 1));
        P.cg_p.alloc(P.esize * std::max<int64_t>(nx, 1));
        if (P.opt.cg_variant == 1) P.cg_ax.alloc(P.esize * std::max<int64_t>(nr, 1));
        P.part_fwd.alloc(std::max<int64_t>(P.fwd.nparts, 1));
        P.part_back.alloc(std::max<int64_t>(P.back.nparts, 1));
        P.part_vec.alloc(kVecBlocks);
        P.tickets.alloc(4);
        MX_CUDA(cudaMemsetAsync(P.tickets.p(), 0, 4 * sizeof(unsigned int), st));
    }
    if (iters > P.scal_iters) {
        MX_CUDA(cudaStreamSynchronize(st));
        P.graphs.clear();
        P.scal.alloc(3 * ((int64_t)iters + 1) + 1);
        MX_CUDA(cudaMemsetAsync(P.scal.p(), 0, 8 * (3 * ((int64_t)iters + 1) + 1), st));
        P.scal_iters = iters;
    }
    if (P.nranks > 1 && !P.comm->capturable()) {  // virtual ranks: eager launches
        cg_enqueue_any(P, y, x, iters, st);
        return;
    }
    auto key = std::make_tuple(y, x, iters, st);
    auto it = P.graphs.find(key);
    if (it == P.graphs.end()) {
        // capture the whole solve once on a private stream, replay it on the caller's stream
        MX_CUDA(cudaStreamSynchronize(st));
        cudaStream_t cap;
        MX_CUDA(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
        cudaGraph_t g = nullptr;
        MX_CUDA(cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal));
        const int64_t before = launch_count();
        try {
            cg_enqueue_any(P, y, x, iters, cap);
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
    MX_CUDA(cudaGraphLaunch(it->second->exec, st));
    count_launch(it->second->nkernels);
    MX_CUDA(cudaGetLastError());
}

void cg_fetch_norms(Plan& P, int32_t iters, double* out, cudaStream_t st) {
    const Scal sc = scal_of(P, (int32_t)P.scal_iters);
    int stop_at = 0;
    MX_CUDA(cudaMemcpyAsync(out, sc.res2, 8 * ((int64_t)iters + 1), cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaMemcpyAsync(&stop_at, sc.stop_at, sizeof(int), cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    for (int32_t k = 0; k <= iters; ++k) {
        if (k >= stop_at) out[k] = out[k - 1];  // iterations that did not run repeat the last norm
        else out[k] = std::sqrt(out[k]);
    }
}

}  // namespace mx
