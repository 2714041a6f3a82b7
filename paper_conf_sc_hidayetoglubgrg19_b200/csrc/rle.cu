// rle.cu -- run-length stage maps (Layout::rle).
//
// The stage map of Listing 3 (buf[i] = x[map[i]]) lists the distinct inputs of a
// partition in stage order; inputs are sorted by Hilbert index (or by slab, then Hilbert index),
// so consecutive map entries are mostly consecutive input indices: mean runs of 19 (config 3)
// and 23 (config-5 shard forward) entries, >= 92 % of the entries in runs of >= 8
// (profiles/r02e_map_runs.jsonl).  The 4 B map entries are 8-10 % of a config-5 forward's bytes.
// Encoding per 32-slot block of a stage (the slots one warp gathers with one instruction):
//   record (int4) = up to 4 runs, run k = start_k | (first slot of the run inside the block << 27)
//   (run 0 starts at slot 0; unused runs have slot 0); a block with more than 4 runs keeps its
//   32 entries in the overflow array and its record holds (1 << 27) | overflow block index.
// Input indices must be < 2^27 (134M: the whole 11293^2 config-5 tomogram fits).
#include "plan.h"

namespace mx {

namespace {

constexpr int kT = 256;
constexpr int32_t kIdxMask = (1 << 27) - 1;

unsigned grid_for(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, kT), 1 << 20)); }

// per stage g of partition p: first map entry and count; blocks per stage
__global__ void stage_span_kernel(const int64_t* __restrict__ stage_base, const int64_t* __restrict__ map_off,
                                  int64_t nparts, int32_t B, int64_t* __restrict__ mstart, int32_t* __restrict__ cnt,
                                  int64_t* __restrict__ nblk) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < nparts; p += (int64_t)gridDim.x * blockDim.x) {
        const int64_t D = map_off[p + 1] - map_off[p];
        for (int64_t g = stage_base[p], s = 0; g < stage_base[p + 1]; ++g, ++s) {
            const int64_t c = min((int64_t)B, D - s * B);
            mstart[g] = map_off[p] + s * B;
            cnt[g] = (int32_t)c;
            nblk[g] = (c + 31) / 32;
        }
    }
}

// one warp per block: runs of consecutive indices inside the block; pass 1 flags overflow
// blocks, pass 2 writes records and overflow entries
template <int kPass>
__global__ void block_runs_kernel(const int32_t* __restrict__ map, const int64_t* __restrict__ mstart,
                                  const int32_t* __restrict__ cnt, const int64_t* __restrict__ blk_base,
                                  int64_t nstages, int64_t nblocks, int64_t* __restrict__ is_ovf,
                                  const int64_t* __restrict__ ovf_pos, int4* __restrict__ rec,
                                  int32_t* __restrict__ ovf) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x / 32);
    for (int64_t b = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32; b < nblocks; b += warps) {
        // stage of block b: largest g with blk_base[g] <= b
        int64_t lo = 0, hi = nstages;
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) >> 1;
            if (blk_base[mid] <= b) lo = mid; else hi = mid;
        }
        const int64_t g = lo;
        const int i = (int)(b - blk_base[g]) * 32 + lane;   // slot inside the stage
        const bool valid = i < cnt[g];
        const int32_t v = valid ? map[mstart[g] + i] : 0;
        const int32_t prev = __shfl_up_sync(0xffffffffu, v, 1);
        const bool start = valid && (lane == 0 || v != prev + 1);
        const unsigned m = __ballot_sync(0xffffffffu, start);
        const int nruns = __popc(m);
        if (kPass == 1) {
            if (lane == 0) is_ovf[b] = nruns > 4 ? 1 : 0;
            continue;
        }
        if (nruns > 4) {
            const int64_t ob = ovf_pos[b];
            ovf[ob * 32 + lane] = v;
            if (lane == 0) rec[b] = make_int4((1 << 27) | (int32_t)ob, 0, 0, 0);
            continue;
        }
        // run q = the (q + 1)-th set bit of m: start value | (slot << 27)
        const int32_t word = start ? (int32_t)((uint32_t)v | ((uint32_t)lane << 27)) : 0;
        int32_t w[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int src = q < nruns ? (int)__fns(m, 0, q + 1) : 0;
            const int32_t got = __shfl_sync(0xffffffffu, word, src);
            w[q] = q < nruns ? got : 0;
        }
        if (lane == 0) rec[b] = make_int4(w[0], w[1], w[2], w[3]);
    }
}

__global__ void max_index_kernel(const int32_t* __restrict__ map, int64_t n, int32_t* __restrict__ out) {
    int32_t mx = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        mx = max(mx, map[i]);
    for (int o = 16; o; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    if ((threadIdx.x & 31) == 0) atomicMax(out, mx);
}

}  // namespace

bool rle_requested() {  // read at every build (tests build both encodings in one process)
    const char* e = std::getenv("MEMXCT_RLE");
    return e ? atoi(e) != 0 : false;
}

bool encode_map_runs(Layout& L, cudaStream_t st) {
    L.rle = false;
    if (L.nstages == 0 || L.nmap == 0) return false;
    {
        DevArr<int32_t> mx;
        mx.alloc(1);
        MX_CUDA(cudaMemsetAsync(mx.p(), 0, 4, st));
        max_index_kernel<<<grid_for(std::min<int64_t>(L.nmap, 1 << 26)), kT, 0, st>>>(L.map.p(), L.nmap, mx.p());
        MX_LAUNCHED();
        int32_t h = 0;
        MX_CUDA(cudaMemcpyAsync(&h, mx.p(), 4, cudaMemcpyDeviceToHost, st));
        MX_CUDA(cudaStreamSynchronize(st));
        if (h > kIdxMask) return false;
    }
    const int64_t ns = L.nstages;
    DevArr<int64_t> mstart, nblk;
    DevArr<int32_t> cnt;
    mstart.alloc(ns);
    nblk.alloc(ns + 1);
    cnt.alloc(ns);
    stage_span_kernel<<<grid_for(L.nparts), kT, 0, st>>>(L.stage_base.p(), L.map_off.p(), L.nparts, L.B, mstart.p(),
                                                          cnt.p(), nblk.p());
    MX_LAUNCHED();
    MX_CUDA(cudaMemsetAsync(nblk.p() + ns, 0, 8, st));
    L.blk_base.alloc(ns + 1);
    exclusive_scan_i64(nblk.p(), L.blk_base.p(), ns + 1, st);
    int64_t nblocks = 0;
    MX_CUDA(cudaMemcpyAsync(&nblocks, L.blk_base.p() + ns, 8, cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    DevArr<int64_t> is_ovf, ovf_pos;
    is_ovf.alloc(nblocks + 1);
    ovf_pos.alloc(nblocks + 1);
    MX_CUDA(cudaMemsetAsync(is_ovf.p() + nblocks, 0, 8, st));
    const unsigned wgrid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(nblocks * 32, kT), 1 << 20));
    block_runs_kernel<1><<<wgrid, kT, 0, st>>>(L.map.p(), mstart.p(), cnt.p(), L.blk_base.p(), ns, nblocks,
                                               is_ovf.p(), nullptr, nullptr, nullptr);
    MX_LAUNCHED();
    exclusive_scan_i64(is_ovf.p(), ovf_pos.p(), nblocks + 1, st);
    MX_CUDA(cudaMemcpyAsync(&L.n_ovf, ovf_pos.p() + nblocks, 8, cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    L.blk_rec.alloc(std::max<int64_t>(nblocks, 1));
    L.ovf.alloc(std::max<int64_t>(L.n_ovf * 32, 1));
    block_runs_kernel<2><<<wgrid, kT, 0, st>>>(L.map.p(), mstart.p(), cnt.p(), L.blk_base.p(), ns, nblocks, nullptr,
                                               ovf_pos.p(), L.blk_rec.p(), L.ovf.p());
    MX_LAUNCHED();
    MX_CUDA(cudaStreamSynchronize(st));
    L.rle = true;
    return true;
}

}  // namespace mx
