// read_peak.cu -- achievable HBM read bandwidth on this GPU for a streaming read shaped like the
// SpMV's matrix stream: 16 B ld.global.nc.L1::no_allocate loads with an L2 evict-first policy,
// one CTA of `threads` per SM slot, several loads in flight per thread.  MEASURED_PEAKS.json's
// hbm_gbs is a read+write copy; a read-only stream is the SpMV's real ceiling.
//
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o read_peak scripts/read_peak.cu
//   ./read_peak [GB=11.6] [reps=20]
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__device__ __forceinline__ uint4 ld_stream(const void* p, uint64_t pol) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(pol));
    return r;
}

// contiguous chunk per CTA (like a partition), U independent 16 B loads per thread per step
template <int U>
__global__ void __launch_bounds__(1024) read_kernel(const uint4* __restrict__ a, int64_t n16, int64_t per_cta, unsigned* out) {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    const int64_t b0 = (int64_t)blockIdx.x * per_cta;
    const int64_t b1 = b0 + per_cta < n16 ? b0 + per_cta : n16;
    unsigned acc = 0;
    for (int64_t i = b0 + threadIdx.x; i < b1; i += (int64_t)U * blockDim.x) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t j = i + (int64_t)u * blockDim.x;
            v[u] = j < b1 ? ld_stream(a + j, pol) : make_uint4(0, 0, 0, 0);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
    if (acc == 0x12345678u) out[0] = acc;
}

// grid-stride interleaved: at any moment all CTAs read neighbouring addresses
template <int U>
__global__ void __launch_bounds__(1024) read_interleaved(const uint4* __restrict__ a, int64_t n16, unsigned* out) {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    const int64_t T = (int64_t)gridDim.x * blockDim.x;
    unsigned acc = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += (int64_t)U * T) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t j = i + (int64_t)u * T;
            v[u] = j < n16 ? ld_stream(a + j, pol) : make_uint4(0, 0, 0, 0);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
    if (acc == 0x12345678u) out[0] = acc;
}

// SpMV-shaped streams: one CTA of 32 warps per "partition", every warp streams `nch` chunks,
// each chunk = 512 B of a 2-byte array (ind) + 1 KB of a 4-byte array (val), 4 chunks unrolled.
// mode 0: warp-private contiguous blocks (the SpMV's SELL layout: warp w's chunks back to back);
// mode 1: chunks of the CTA's 32 warps interleaved (chunk c of warp w at c * 32 + w).
template <int MODE>
__global__ void __launch_bounds__(1024) spmv_shape_kernel(const uint4* __restrict__ ind, const uint4* __restrict__ val,
                                                          int nch, unsigned* out) {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t cta0 = (int64_t)blockIdx.x * 32 * nch;  // chunk index base of this CTA
    unsigned acc = 0;
#pragma unroll 4
    for (int c = 0; c < nch; ++c) {
        const int64_t ch = MODE == 0 ? cta0 + (int64_t)warp * nch + c : cta0 + (int64_t)c * 32 + warp;
        const uint4 a = ld_stream(ind + ch * 32 + lane, pol);
        const uint4 b = ld_stream(val + ch * 64 + lane, pol);
        const uint4 d = ld_stream(val + ch * 64 + 32 + lane, pol);
        acc ^= a.x ^ b.y ^ d.z ^ a.w ^ b.x ^ d.w;
    }
    if (acc == 0x12345678u) out[0] = acc;
}

template <int MODE>
void run_shape(const uint4* a, int64_t n16, int ctas, unsigned* out, int reps) {
    // split the buffer: ind third, val two thirds
    const int64_t chunks = n16 / 96;  // 96 x 16 B = 1.5 KB per chunk
    const int nch = (int)(chunks / ((int64_t)ctas * 32));
    const uint4* ind = a;
    const uint4* val = a + (int64_t)ctas * 32 * nch * 32;
    const double bytes = (double)ctas * 32 * nch * 1536.0;
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    for (int w = 0; w < 2; ++w) spmv_shape_kernel<MODE><<<ctas, 1024>>>(ind, val, nch, out);
    CK(cudaEventRecord(e0));
    for (int r = 0; r < reps; ++r) spmv_shape_kernel<MODE><<<ctas, 1024>>>(ind, val, nch, out);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    CK(cudaGetLastError());
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    ms /= reps;
    printf("{\"mode\": \"spmv_shape_%s\", \"ctas\": %d, \"chunks_per_warp\": %d, \"ms\": %.4f, \"GBs\": %.1f}\n",
           MODE == 0 ? "warp_private" : "cta_interleaved", ctas, nch, ms, bytes / (ms * 1e6));
}

template <int U>
void run_il(const uint4* a, int64_t n16, int ctas, int threads, unsigned* out, int reps, double bytes) {
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    for (int w = 0; w < 3; ++w) read_interleaved<U><<<ctas, threads>>>(a, n16, out);
    CK(cudaEventRecord(e0));
    for (int r = 0; r < reps; ++r) read_interleaved<U><<<ctas, threads>>>(a, n16, out);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    ms /= reps;
    printf("{\"mode\": \"interleaved\", \"ctas\": %d, \"threads\": %d, \"U\": %d, \"ms\": %.4f, \"GBs\": %.1f}\n",
           ctas, threads, U, ms, bytes / (ms * 1e6));
}

template <int U>
void run(const uint4* a, int64_t n16, int ctas, int threads, unsigned* out, int reps, double bytes) {
    const int64_t per = (n16 + ctas - 1) / ctas;
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    for (int w = 0; w < 3; ++w) read_kernel<U><<<ctas, threads>>>(a, n16, per, out);
    CK(cudaEventRecord(e0));
    for (int r = 0; r < reps; ++r) read_kernel<U><<<ctas, threads>>>(a, n16, per, out);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    ms /= reps;
    printf("{\"ctas\": %d, \"threads\": %d, \"U\": %d, \"ms\": %.4f, \"GBs\": %.1f}\n", ctas, threads, U, ms,
           bytes / (ms * 1e6));
}

int main(int argc, char** argv) {
    const double gb = argc > 1 ? atof(argv[1]) : 11.6;
    const int reps = argc > 2 ? atoi(argv[2]) : 20;
    const int64_t n16 = (int64_t)(gb * 1e9 / 16);
    int sms = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    uint4* a;
    unsigned* out;
    CK(cudaMalloc(&a, n16 * 16));
    CK(cudaMalloc(&out, 4));
    CK(cudaMemset(a, 1, n16 * 16));
    const double bytes = (double)n16 * 16;
    // one persistent wave (1 CTA of 1024 per SM, the SpMV's shape), and many-wave grids
    run<4>(a, n16, sms, 1024, out, reps, bytes);
    run<8>(a, n16, sms, 1024, out, reps, bytes);
    run<4>(a, n16, 2 * sms, 512, out, reps, bytes);
    run<8>(a, n16, 2 * sms, 512, out, reps, bytes);
    run<4>(a, n16, 1500, 1024, out, reps, bytes);
    run<4>(a, n16, 16 * sms, 256, out, reps, bytes);
    run<8>(a, n16, 16 * sms, 256, out, reps, bytes);
    run<4>(a, n16, 64 * sms, 256, out, reps, bytes);
    run<16>(a, n16, sms, 1024, out, reps, bytes);
    run<16>(a, n16, 8 * sms, 256, out, reps, bytes);
    run_il<4>(a, n16, sms, 1024, out, reps, bytes);
    run_il<8>(a, n16, sms, 1024, out, reps, bytes);
    run_il<16>(a, n16, sms, 1024, out, reps, bytes);
    run_il<8>(a, n16, 8 * sms, 256, out, reps, bytes);
    run_il<16>(a, n16, 8 * sms, 256, out, reps, bytes);
    run_il<4>(a, n16, 4 * sms, 512, out, reps, bytes);
    run_shape<0>(a, n16, 1500, out, reps);
    run_shape<1>(a, n16, 1500, out, reps);
    run_shape<0>(a, n16, 148, out, reps);
    run_shape<1>(a, n16, 148, out, reps);
    run_shape<0>(a, n16, 4440, out, reps);
    run_shape<1>(a, n16, 4440, out, reps);
    return 0;
}
