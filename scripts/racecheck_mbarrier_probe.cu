// Does compute-sanitizer racecheck model mbarrier arrive / try_wait.parity synchronisation?
// The drifting-stage SpMV (spmv.cu: spmv_f32_drift_kernel) reuses three shared stage buffers
// behind two mbarrier rings; racecheck reports write(gather)/read(stream) hazards on them.  This
// probe runs the SAME protocol, stripped to the buffer handoff, in three variants:
//   mode 0  the drift protocol (full / done rings, warp arrivals after __syncwarp)
//   mode 1  the same with a __syncthreads() before every gather (racecheck's native barrier)
//   mode 2  a real race: the wait on `done` before the gather is removed
// and checks the result on the host; argument 2 = 1 adds per-warp delays so a broken handoff
// shows up as wrong sums (r02e: racecheck reports hazards for all three modes alike).  nvcc -gencode arch=compute_100a,code=sm_100a -o probe probe.cu
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, unsigned parity) {
    for (;;) {
        uint32_t ok;
        asm volatile("{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\t"
                     "selp.u32 %0, 1, 0, P;\n\t}" : "=r"(ok) : "r"(smem_addr(b)), "r"(parity) : "memory");
        if (ok) return;
    }
}

constexpr int B = 256;
__global__ void probe(const float* __restrict__ x, int ns, int mode, float* out, int jitter) {
    __shared__ float buf[3][B];
    __shared__ __align__(8) uint64_t full[3], done[3];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
    if (threadIdx.x == 0)
        for (int b = 0; b < 3; ++b) { mbar_init(&full[b], nw); mbar_init(&done[b], nw); }
    __syncthreads();
    auto gather = [&](int s) {
        for (int i = threadIdx.x; i < B; i += blockDim.x) buf[s % 3][i] = x[s * B + i];
        __syncwarp();
        if (lane == 0) mbar_arrive(&full[s % 3]);
    };
    gather(0);
    if (ns > 1) gather(1);
    float acc = 0.f;
    for (int s = 0; s < ns; ++s) {
        mbar_wait(&full[s % 3], (s / 3) & 1);
        if (jitter && ((warp * 7 + s) % 5 == 0)) __nanosleep(2000 + 131 * warp);
        for (int i = lane; i < B; i += 32) acc += buf[s % 3][(i * 7 + warp) % B];   // read other warps' slots
        __syncwarp();
        if (lane == 0) mbar_arrive(&done[s % 3]);
        if (s + 2 < ns) {
            if (mode == 1) __syncthreads();
            if (mode != 2 && s >= 1) mbar_wait(&done[(s + 2) % 3], ((s - 1) / 3) & 1);
            gather(s + 2);
        }
    }
    out[threadIdx.x] = acc;
}

int main(int argc, char** argv) {
    const int mode = argc > 1 ? atoi(argv[1]) : 0, jitter = argc > 2 ? atoi(argv[2]) : 0, ns = 12, nt = 256;
    float *x, *out;
    cudaMallocManaged(&x, sizeof(float) * ns * B);
    cudaMallocManaged(&out, sizeof(float) * nt);
    for (int i = 0; i < ns * B; ++i) x[i] = (float)(i % 97);
    probe<<<1, nt>>>(x, ns, mode, out, jitter);
    cudaDeviceSynchronize();
    // expected: every thread sums 8 reads per stage of its warp's slots
    int bad = 0;
    for (int t = 0; t < nt; ++t) {
        const int warp = t >> 5, lane = t & 31;
        float e = 0.f;
        for (int s = 0; s < ns; ++s)
            for (int i = lane; i < B; i += 32) e += x[s * B + (i * 7 + warp) % B];
        bad += (out[t] != e);
    }
    printf("mode %d jitter %d: %s (%d threads wrong)\n", mode, jitter, bad ? "WRONG" : "correct", bad);
    return 0;
}
