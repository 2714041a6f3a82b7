// trace.cu -- Siddon ray tracing on the device (sec. 2.3; build step (2) of P:838-845).
//
// One thread per ray; rays are visited in plan (Hilbert) order so a warp traces 32 neighbouring
// rays of one Hilbert tile (similar chords, little divergence).  Geometry follows readings R1-R4:
//   theta_m = m*pi/M (host cos/sin tables), t_k = (k + 1/2) - C/2, grid [-N/2, N/2]^2 of unit
//   pixels, line p(a) = t (cos, sin) + a (-sin, cos).
// The ray is clipped to the grid ([lo, hi]); the x-line and y-line crossings strictly inside
// (lo, hi) are each monotone in the line index, so instead of sorting all candidates we MERGE the
// two monotone streams, drop exact duplicates, and emit one segment per consecutive pair longer
// than EPS_LEN, assigned to the pixel containing its midpoint.
//
// All fp64 arithmetic uses explicit round-to-nearest intrinsics and this file is compiled with
// --fmad=false, so every parameter, midpoint and length is the correctly rounded value of the
// expression written in DESIGN.md (reading R4): no contraction into FMAs.
#include <cmath>

#include "plan.h"

namespace mx {

namespace {

constexpr double kEpsDir = 1e-15;
constexpr double kEpsLen = 1e-9;

// Stream of crossing parameters of the grid lines q = 0..N along one axis, in ascending order,
// restricted to the open interval (lo, hi).
struct Crossings {
    double p0, d, L;
    int32_t q, qend, step;  // next line index, one-past-last, direction
    bool active;
    __device__ void init(double p0_, double d_, double L_, int32_t n, bool use) {
        p0 = p0_; d = d_; L = L_; active = use;
        if (d > 0) { q = 0; qend = n + 1; step = 1; } else { q = n; qend = -1; step = -1; }
    }
    __device__ __forceinline__ double at(int32_t qq) const {
        return __ddiv_rn(__dsub_rn(__dsub_rn((double)qq, L), p0), d);
    }
    // next value > lo and < hi, or +inf when exhausted
    __device__ __forceinline__ double next(double lo, double hi) {
        while (active && q != qend) {
            const double a = at(q);
            q += step;
            if (a <= lo) continue;
            if (a < hi) return a;
            active = false;  // monotone: every later line is >= hi as well
        }
        active = false;
        return INFINITY;
    }
};

template <bool kEmit>
__device__ int64_t trace_one(int32_t n, int32_t c_chan, int64_t ray, double cs, double sn,
                             const int32_t* __restrict__ pix_rank, uint32_t* __restrict__ cols,
                             float* __restrict__ vals) {
    const int64_t k = ray % c_chan;
    const double L = __ddiv_rn((double)n, 2.0);
    const double t = __dsub_rn(__dadd_rn((double)k, 0.5), __ddiv_rn((double)c_chan, 2.0));
    const double p0x = __dmul_rn(t, cs), p0y = __dmul_rn(t, sn);
    const double dx = -sn, dy = cs;
    double lo = -INFINITY, hi = INFINITY;
    const bool ux = fabs(dx) >= kEpsDir, uy = fabs(dy) >= kEpsDir;
    if (!ux) { if (!(-L < p0x && p0x < L)) return 0; }
    else {
        const double t1 = __ddiv_rn(__dsub_rn(-L, p0x), dx), t2 = __ddiv_rn(__dsub_rn(L, p0x), dx);
        lo = fmax(lo, fmin(t1, t2));
        hi = fmin(hi, fmax(t1, t2));
    }
    if (!uy) { if (!(-L < p0y && p0y < L)) return 0; }
    else {
        const double t1 = __ddiv_rn(__dsub_rn(-L, p0y), dy), t2 = __ddiv_rn(__dsub_rn(L, p0y), dy);
        lo = fmax(lo, fmin(t1, t2));
        hi = fmin(hi, fmax(t1, t2));
    }
    if (__dsub_rn(hi, lo) <= kEpsLen) return 0;

    Crossings X, Y;
    X.init(p0x, dx, L, n, ux);
    Y.init(p0y, dy, L, n, uy);
    double ax = X.next(lo, hi), ay = Y.next(lo, hi);
    double prev = lo;
    int64_t cnt = 0;
    for (;;) {
        double v;
        bool last = false;
        if (ax <= ay) { v = ax; ax = X.next(lo, hi); } else { v = ay; ay = Y.next(lo, hi); }
        if (v == INFINITY) { v = hi; last = true; }
        if (v != prev) {
            const double seg = __dsub_rn(v, prev);
            if (seg > kEpsLen) {
                if (kEmit) {
                    const double mid = __ddiv_rn(__dadd_rn(prev, v), 2.0);
                    const double fx = __dadd_rn(__dadd_rn(p0x, __dmul_rn(mid, dx)), L);
                    const double fy = __dadd_rn(__dadd_rn(p0y, __dmul_rn(mid, dy)), L);
                    int64_t j = (int64_t)floor(fx), i = (int64_t)floor(fy);
                    j = j < 0 ? 0 : (j > n - 1 ? n - 1 : j);
                    i = i < 0 ? 0 : (i > n - 1 ? n - 1 : i);
                    cols[cnt] = (uint32_t)pix_rank[i * n + j];
                    vals[cnt] = __double2float_rn(seg);
                }
                ++cnt;
            }
            prev = v;
        }
        if (last) break;
    }
    return cnt;
}

__global__ void trace_count_kernel(int32_t n, int32_t c_chan, int64_t nrays,
                                   const int32_t* __restrict__ ray_of_row,
                                   const double* __restrict__ cos_t, const double* __restrict__ sin_t,
                                   int32_t* __restrict__ row_len) {
    const int64_t h = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (h >= nrays) return;
    const int64_t ray = ray_of_row[h];
    const int64_t m = ray / c_chan;
    row_len[h] = (int32_t)trace_one<false>(n, c_chan, ray, cos_t[m], sin_t[m], nullptr, nullptr, nullptr);
}

__global__ void trace_emit_kernel(int32_t n, int32_t c_chan, int64_t nrays,
                                  const int32_t* __restrict__ ray_of_row,
                                  const double* __restrict__ cos_t, const double* __restrict__ sin_t,
                                  const int32_t* __restrict__ pix_rank, const int64_t* __restrict__ row_ptr,
                                  uint32_t* __restrict__ cols, float* __restrict__ vals,
                                  uint32_t* __restrict__ row_ids) {
    const int64_t h = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (h >= nrays) return;
    const int64_t ray = ray_of_row[h];
    const int64_t m = ray / c_chan;
    const int64_t b = row_ptr[h];
    const int64_t cnt = trace_one<true>(n, c_chan, ray, cos_t[m], sin_t[m], pix_rank, cols + b, vals + b);
    for (int64_t e = 0; e < cnt; ++e) row_ids[b + e] = (uint32_t)h;
}

}  // namespace

void trace_count(const Plan& P, const double* cos_t, const double* sin_t, int64_t nrays,
                 int32_t* row_len, cudaStream_t st) {
    if (nrays == 0) return;
    const int threads = 128;
    trace_count_kernel<<<(unsigned)ceil_div(nrays, threads), threads, 0, st>>>(
        P.n, P.c, nrays, P.sino_nat_of_h.p(), cos_t, sin_t, row_len);
    MX_LAUNCHED();
}

void trace_emit(const Plan& P, const double* cos_t, const double* sin_t, int64_t nrays,
                const int64_t* row_ptr, uint32_t* cols, float* vals, uint32_t* row_ids,
                cudaStream_t st) {
    if (nrays == 0) return;
    const int threads = 128;
    trace_emit_kernel<<<(unsigned)ceil_div(nrays, threads), threads, 0, st>>>(
        P.n, P.c, nrays, P.sino_nat_of_h.p(), cos_t, sin_t, P.tomo_h_of_nat.p(), row_ptr, cols,
        vals, row_ids);
    MX_LAUNCHED();
}

}  // namespace mx
