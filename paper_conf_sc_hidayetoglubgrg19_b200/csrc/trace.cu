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

// Modes: kCount (segments), kEmit (write Hilbert pixel - lo and fp32 length), kHist (atomicAdd 1
// per segment into hist[Hilbert pixel]).  kFilter keeps only segments whose Hilbert pixel index
// lies in [lo, hi) -- the local tomogram subdomain of a rank (P > 1, A_p of P:758-811).
enum Mode { kCount = 0, kEmit = 1, kHist = 2 };

template <int kMode, bool kFilter>
__device__ int64_t trace_one(int32_t n, int32_t c_chan, int64_t ray, double cs, double sn,
                             const int32_t* __restrict__ pix_rank, int64_t lo, int64_t hi,
                             uint32_t* __restrict__ cols, float* __restrict__ vals,
                             int32_t* __restrict__ hist) {
    const int64_t k = ray % c_chan;
    const double L = __ddiv_rn((double)n, 2.0);
    const double t = __dsub_rn(__dadd_rn((double)k, 0.5), __ddiv_rn((double)c_chan, 2.0));
    const double p0x = __dmul_rn(t, cs), p0y = __dmul_rn(t, sn);
    const double dx = -sn, dy = cs;
    double lo_a = -INFINITY, hi_a = INFINITY;
    const bool ux = fabs(dx) >= kEpsDir, uy = fabs(dy) >= kEpsDir;
    if (!ux) { if (!(-L < p0x && p0x < L)) return 0; }
    else {
        const double t1 = __ddiv_rn(__dsub_rn(-L, p0x), dx), t2 = __ddiv_rn(__dsub_rn(L, p0x), dx);
        lo_a = fmax(lo_a, fmin(t1, t2));
        hi_a = fmin(hi_a, fmax(t1, t2));
    }
    if (!uy) { if (!(-L < p0y && p0y < L)) return 0; }
    else {
        const double t1 = __ddiv_rn(__dsub_rn(-L, p0y), dy), t2 = __ddiv_rn(__dsub_rn(L, p0y), dy);
        lo_a = fmax(lo_a, fmin(t1, t2));
        hi_a = fmin(hi_a, fmax(t1, t2));
    }
    if (__dsub_rn(hi_a, lo_a) <= kEpsLen) return 0;

    Crossings X, Y;
    X.init(p0x, dx, L, n, ux);
    Y.init(p0y, dy, L, n, uy);
    double ax = X.next(lo_a, hi_a), ay = Y.next(lo_a, hi_a);
    double prev = lo_a;
    int64_t cnt = 0;
    constexpr bool kNeedPixel = (kMode != kCount) || kFilter;
    for (;;) {
        double v;
        bool last = false;
        if (ax <= ay) { v = ax; ax = X.next(lo_a, hi_a); } else { v = ay; ay = Y.next(lo_a, hi_a); }
        if (v == INFINITY) { v = hi_a; last = true; }
        if (v != prev) {
            const double seg = __dsub_rn(v, prev);
            if (seg > kEpsLen) {
                int64_t h = 0;
                if (kNeedPixel) {
                    const double mid = __ddiv_rn(__dadd_rn(prev, v), 2.0);
                    const double fx = __dadd_rn(__dadd_rn(p0x, __dmul_rn(mid, dx)), L);
                    const double fy = __dadd_rn(__dadd_rn(p0y, __dmul_rn(mid, dy)), L);
                    int64_t j = (int64_t)floor(fx), i = (int64_t)floor(fy);
                    j = j < 0 ? 0 : (j > n - 1 ? n - 1 : j);
                    i = i < 0 ? 0 : (i > n - 1 ? n - 1 : i);
                    h = pix_rank[i * n + j];
                }
                if (!kFilter || (h >= lo && h < hi)) {
                    if (kMode == kEmit) {
                        cols[cnt] = (uint32_t)(h - lo);
                        vals[cnt] = __double2float_rn(seg);
                    }
                    if (kMode == kHist) atomicAdd(hist + (h - lo), 1);
                    ++cnt;
                }
            }
            prev = v;
        }
        if (last) break;
    }
    return cnt;
}

// absolute row r: Hilbert ray hray[r] (footprint list) or r itself; natural ray = nat_of_h[...]
__device__ __forceinline__ int64_t natural_ray(const int32_t* __restrict__ hray, int64_t, int64_t r,
                                               const int32_t* __restrict__ nat_of_h) {
    return nat_of_h[hray ? (int64_t)hray[r] : r];
}

template <bool kFilter>
__global__ void trace_count_kernel(int32_t n, int32_t c_chan, int64_t r0, int64_t nrows,
                                   const int32_t* __restrict__ hray, const int32_t* __restrict__ nat_of_h,
                                   const double* __restrict__ cos_t, const double* __restrict__ sin_t,
                                   const int32_t* __restrict__ pix_rank, int64_t lo, int64_t hi,
                                   int32_t* __restrict__ row_len) {
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= nrows) return;
    const int64_t ray = natural_ray(hray, r0, r0 + r, nat_of_h);
    const int64_t m = ray / c_chan;
    row_len[r] = (int32_t)trace_one<kCount, kFilter>(n, c_chan, ray, cos_t[m], sin_t[m], pix_rank, lo, hi,
                                                      nullptr, nullptr, nullptr);
}

__global__ void trace_emit_kernel(int32_t n, int32_t c_chan, int64_t r0, int64_t nrows,
                                  const int32_t* __restrict__ hray, const int32_t* __restrict__ nat_of_h,
                                  const double* __restrict__ cos_t, const double* __restrict__ sin_t,
                                  const int32_t* __restrict__ pix_rank, int64_t lo, int64_t hi,
                                  const int64_t* __restrict__ row_ptr, uint32_t* __restrict__ cols,
                                  float* __restrict__ vals, uint32_t* __restrict__ row_ids) {
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= nrows) return;
    const int64_t ray = natural_ray(hray, r0, r0 + r, nat_of_h);
    const int64_t m = ray / c_chan;
    const int64_t b = row_ptr[r];
    const int64_t cnt = trace_one<kEmit, true>(n, c_chan, ray, cos_t[m], sin_t[m], pix_rank, lo, hi, cols + b,
                                               vals + b, nullptr);
    for (int64_t e = 0; e < cnt; ++e) row_ids[b + e] = (uint32_t)(r0 + r);
}

template <bool kFilter>
__global__ void trace_hist_kernel(int32_t n, int32_t c_chan, int64_t r0, int64_t nrows,
                                  const int32_t* __restrict__ hray, const int32_t* __restrict__ nat_of_h,
                                  const double* __restrict__ cos_t, const double* __restrict__ sin_t,
                                  const int32_t* __restrict__ pix_rank, int64_t lo, int64_t hi,
                                  int32_t* __restrict__ hist) {
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= nrows) return;
    const int64_t ray = natural_ray(hray, r0, r0 + r, nat_of_h);
    const int64_t m = ray / c_chan;
    trace_one<kHist, kFilter>(n, c_chan, ray, cos_t[m], sin_t[m], pix_rank, lo, hi, nullptr, nullptr, hist);
}

}  // namespace

void trace_count(const Plan& P, const Geometry& G, const int32_t* hray, int64_t r0, int64_t nrows, int64_t lo,
                 int64_t hi, bool filter, int32_t* row_len, cudaStream_t st) {
    if (nrows == 0) return;
    const int threads = 128;
    const unsigned blocks = (unsigned)ceil_div(nrows, threads);
    if (filter)
        trace_count_kernel<true><<<blocks, threads, 0, st>>>(P.n, P.c, r0, nrows, hray, P.sino_nat_of_h.p(),
                                                             G.cos_t, G.sin_t, P.tomo_h_of_nat.p(), lo, hi, row_len);
    else
        trace_count_kernel<false><<<blocks, threads, 0, st>>>(P.n, P.c, r0, nrows, hray, P.sino_nat_of_h.p(),
                                                              G.cos_t, G.sin_t, P.tomo_h_of_nat.p(), lo, hi, row_len);
    MX_LAUNCHED();
}

void trace_emit(const Plan& P, const Geometry& G, const int32_t* hray, int64_t r0, int64_t nrows, int64_t lo,
                int64_t hi, const int64_t* row_ptr, uint32_t* cols, float* vals, uint32_t* row_ids,
                cudaStream_t st) {
    if (nrows == 0) return;
    const int threads = 128;
    trace_emit_kernel<<<(unsigned)ceil_div(nrows, threads), threads, 0, st>>>(
        P.n, P.c, r0, nrows, hray, P.sino_nat_of_h.p(), G.cos_t, G.sin_t, P.tomo_h_of_nat.p(), lo, hi, row_ptr,
        cols, vals, row_ids);
    MX_LAUNCHED();
}

void trace_hist(const Plan& P, const Geometry& G, const int32_t* hray, int64_t r0, int64_t nrows, int64_t lo,
                int64_t hi, bool filter, int32_t* hist, cudaStream_t st) {
    if (nrows <= 0) return;
    const int threads = 128;
    const unsigned blocks = (unsigned)ceil_div(nrows, threads);
    if (filter)
        trace_hist_kernel<true><<<blocks, threads, 0, st>>>(P.n, P.c, r0, nrows, hray, P.sino_nat_of_h.p(), G.cos_t,
                                                            G.sin_t, P.tomo_h_of_nat.p(), lo, hi, hist);
    else
        trace_hist_kernel<false><<<blocks, threads, 0, st>>>(P.n, P.c, r0, nrows, hray, P.sino_nat_of_h.p(),
                                                             G.cos_t, G.sin_t, P.tomo_h_of_nat.p(), 0, 0, hist);
    MX_LAUNCHED();
}

}  // namespace mx
