// sirt.cu -- SIRT on the same memoized operators (the solver the paper runs
// for its one-to-one comparison with Trace, 45 iterations).
//
//   x_0 = 0;  x_{k+1} = x_k + C A^T R (y - A x_k),
//   R = diag(1 / row sums of A), C = diag(1 / column sums of A)   (0 where a sum is 0),
// the textbook simultaneous iterative reconstruction technique.  Row and column sums are
// projections of all-ones vectors with the plan's own kernels (so at P > 1 they include the
// exchange).  res[k] = ||y - A x_k|| (the forward projection of every iteration computes it).
#include "plan.h"

namespace mx {

namespace {

constexpr int kT = 256;

unsigned nb(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, kT), 4 * num_sms())); }

template <class T> __global__ void fill_kernel(T* v, int64_t n, T a) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) v[i] = a;
}

template <class T> __global__ void invert_kernel(T* v, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        v[i] = v[i] != T(0) ? T(1) / v[i] : T(0);
}

// r = R (y - ax); partial of ||y - ax||^2 per block (fixed grid: deterministic)
template <class T>
__global__ void __launch_bounds__(kT)
residual_kernel(const T* __restrict__ y, const T* __restrict__ ax, const T* __restrict__ rinv, T* __restrict__ r,
                int64_t n, double* __restrict__ part) {
    __shared__ double red[kT / 32];
    double acc = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * kT + threadIdx.x; i < n; i += (int64_t)gridDim.x * kT) {
        const T e = y[i] - ax[i];
        r[i] = e * rinv[i];
        acc += (double)e * (double)e;
    }
    for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        double s = 0.0;
        for (int w = 0; w < kT / 32; ++w) s += red[w];
        part[blockIdx.x] = s;
    }
}

// sequential sum of the block partials (one thread, fixed order)
__global__ void sum_parts_kernel(const double* __restrict__ part, int n, double* out) {
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        double s = 0.0;
        for (int i = 0; i < n; ++i) s += part[i];
        *out = s;
    }
}

// x += C s
template <class T>
__global__ void update_kernel(T* __restrict__ x, const T* __restrict__ s, const T* __restrict__ cinv, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] += cinv[i] * s[i];
}

template <class T>
void sirt_t(Plan& P, const T* y, T* x, int32_t iters, double* res2_dev, cudaStream_t st) {
    const int64_t nx = P.local_len(0), nr = P.local_len(1);
    auto& S = P.sirt;
    if (!S.ready) {
        S.rinv.alloc(P.esize * std::max<int64_t>(nr, 1));
        S.cinv.alloc(P.esize * std::max<int64_t>(nx, 1));
        S.r.alloc(P.esize * std::max<int64_t>(nr, 1));
        S.ax.alloc(P.esize * std::max<int64_t>(nr, 1));
        S.s.alloc(P.esize * std::max<int64_t>(nx, 1));
        S.ones.alloc(P.esize * std::max<int64_t>(std::max(nx, nr), 1));
        S.part.alloc(4 * num_sms());
        fill_kernel<T><<<nb(std::max(nx, nr)), kT, 0, st>>>(S.ones.as<T>(), std::max(nx, nr), T(1));
        MX_LAUNCHED();
        apply_forward(P, S.ones.get(), S.rinv.get(), st);  // row sums of A
        apply_back(P, S.ones.get(), S.cinv.get(), st);     // column sums of A
        invert_kernel<T><<<nb(nr), kT, 0, st>>>(S.rinv.as<T>(), nr);
        MX_LAUNCHED();
        invert_kernel<T><<<nb(nx), kT, 0, st>>>(S.cinv.as<T>(), nx);
        MX_LAUNCHED();
        S.ready = true;
    }
    fill_kernel<T><<<nb(nx), kT, 0, st>>>(x, nx, T(0));
    MX_LAUNCHED();
    for (int32_t k = 0; k <= iters; ++k) {
        apply_forward(P, x, S.ax.get(), st);                                       // A x_k
        const unsigned g = nb(nr);
        residual_kernel<T><<<g, kT, 0, st>>>(y, S.ax.as<T>(), S.rinv.as<T>(), S.r.as<T>(), nr, S.part.p());
        MX_LAUNCHED();
        sum_parts_kernel<<<1, 32, 0, st>>>(S.part.p(), (int)g, res2_dev + k);       // ||y - A x_k||^2
        MX_LAUNCHED();
        if (P.dist) P.comm->allreduce_sum(res2_dev + k, 1, DType::F64, st);
        if (k == iters) break;
        apply_back(P, S.r.get(), S.s.get(), st);                                    // A^T R (y - A x_k)
        update_kernel<T><<<nb(nx), kT, 0, st>>>(x, S.s.as<T>(), S.cinv.as<T>(), nx);
        MX_LAUNCHED();
    }
}

}  // namespace

void sirt_run(Plan& P, const void* y, void* x, int32_t iters, double* residual_norms, cudaStream_t st) {
    DevArr<double> res2;
    res2.alloc(iters + 1);
    if (P.esize == 4) sirt_t<float>(P, (const float*)y, (float*)x, iters, res2.p(), st);
    else sirt_t<double>(P, (const double*)y, (double*)x, iters, res2.p(), st);
    std::vector<double> h(iters + 1);
    MX_CUDA(cudaMemcpyAsync(h.data(), res2.p(), 8 * (iters + 1), cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    if (residual_norms)
        for (int32_t k = 0; k <= iters; ++k) residual_norms[k] = std::sqrt(h[k]);
}

}  // namespace mx
