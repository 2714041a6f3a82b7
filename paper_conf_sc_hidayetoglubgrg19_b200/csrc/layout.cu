// layout.cu -- preprocessing: Siddon-traced A, order-preserving transposition to
// A^T, and the multi-stage buffered layout of both matrices, all on the device.
//
// Pipeline (build_matrices):
//   1. count pass: row lengths of A over rays in Hilbert order (trace.cu), exclusive scan;
//   2. emit pass: (Hilbert pixel, fp32 length, Hilbert ray) per entry, rows in Hilbert order;
//   3. A^T by a STABLE radix sort on the pixel key: entries of each pixel keep ascending ray
//      order -- the scan-based, order-preserving transposition of P:847-858 (no atomics);
//   4. A with ascending pixel order inside each ray by a second stable sort (on the ray key) of
//      the A^T entries;
//   5. build_layout for each direction.
//
// build_layout (per direction), reading R10/R11:
//   * partition p = R consecutive Hilbert rows (one CTA); its distinct inputs are found with a
//     per-partition bitmap over the input domain; a popcount prefix over the bitmap gives every
//     entry the rank of its input among the partition's distinct inputs, in ascending Hilbert
//     order (the stage map order);
//   * stage s of p = ranks [s*B, (s+1)*B): map[s*B + i] = input index (P:598-599, 16-bit local
//     index i = rank % B);
//   * per 32-row slice and stage: width = max entries of its rows in that stage, rounded up to
//     kVec; slots stored column-chunk-major (plan.h) and padded with (ind 0, val 0).
#include <cub/block/block_scan.cuh>
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <cmath>
#include <vector>

#include "plan.h"

namespace mx {

namespace {

constexpr int kThreads = 256;

inline unsigned blocks_for(int64_t n, int threads = kThreads) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, threads), 1 << 30));
}

template <class T> __global__ void iota_kernel(T* out, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (T)i;
}

__global__ void widen_kernel(const int32_t* in, int64_t* out, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = in[i];
}

// row_ptr[r] = first entry with row_ids >= r (row_ids sorted ascending), r in [0, nrows]
__global__ void row_ptr_kernel(const uint32_t* __restrict__ row_ids, int64_t nnz, int64_t nrows,
                               int64_t* __restrict__ row_ptr) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r <= nrows; r += (int64_t)gridDim.x * blockDim.x) {
        int64_t lo = 0, hi = nnz;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if ((int64_t)row_ids[mid] < r) lo = mid + 1; else hi = mid;
        }
        row_ptr[r] = lo;
    }
}

// mark the input of every entry of partitions [pa, pb) in the chunk bitmap
__global__ void mark_kernel(const uint32_t* __restrict__ row_ids, const uint32_t* __restrict__ cols,
                            int64_t e0, int64_t e1, int32_t R, int64_t pa, int64_t words,
                            uint32_t* __restrict__ bitmap) {
    for (int64_t e = e0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < e1; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t p = row_ids[e] / R - pa;
        const uint32_t c = cols[e];
        atomicOr(bitmap + p * words + (c >> 5), 1u << (c & 31));
    }
}

// per partition: exclusive popcount prefix of its bitmap words, and its distinct count
constexpr int kScanThreads = 512;
__global__ void __launch_bounds__(kScanThreads)
prefix_kernel(const uint32_t* __restrict__ bitmap, int64_t words, int64_t pa,
              uint32_t* __restrict__ word_prefix, int64_t* __restrict__ distinct) {
    using Scan = cub::BlockScan<uint32_t, kScanThreads>;
    __shared__ typename Scan::TempStorage tmp;
    const int64_t p = blockIdx.x;
    const uint32_t* bm = bitmap + p * words;
    uint32_t* wp = word_prefix + p * words;
    uint32_t carry = 0;
    for (int64_t w0 = 0; w0 < words; w0 += kScanThreads) {
        const int64_t w = w0 + threadIdx.x;
        const uint32_t v = (w < words) ? (uint32_t)__popc(bm[w]) : 0u;
        uint32_t ex, tot;
        Scan(tmp).ExclusiveSum(v, ex, tot);
        if (w < words) wp[w] = carry + ex;
        carry += tot;
        __syncthreads();
    }
    if (threadIdx.x == 0) distinct[pa + p] = carry;
}

__global__ void rank_kernel(const uint32_t* __restrict__ row_ids, const uint32_t* __restrict__ cols,
                            int64_t e0, int64_t e1, int32_t R, int64_t pa, int64_t words,
                            const uint32_t* __restrict__ bitmap, const uint32_t* __restrict__ word_prefix,
                            uint32_t* __restrict__ rank) {
    for (int64_t e = e0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < e1; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t p = row_ids[e] / R - pa;
        const uint32_t c = cols[e];
        const int64_t w = p * words + (c >> 5);
        rank[e] = word_prefix[w] + (uint32_t)__popc(bitmap[w] & ((1u << (c & 31)) - 1u));
    }
}

// map[map_off[p] + rank] = translated input of every set bit of partition p's bitmap
__global__ void map_kernel(const uint32_t* __restrict__ bitmap, const uint32_t* __restrict__ word_prefix,
                           int64_t words, int64_t nchunk, int64_t pa, const int64_t* __restrict__ map_off,
                           const int32_t* __restrict__ translate, int32_t* __restrict__ map) {
    const int64_t total = nchunk * words;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t b = bitmap[i];
        if (!b) continue;
        const int64_t p = i / words, w = i % words;
        int64_t r = map_off[pa + p] + word_prefix[i];
        while (b) {
            const int bit = __ffs(b) - 1;
            b &= b - 1;
            const int64_t col = w * 32 + bit;
            map[r++] = translate ? translate[col] : (int32_t)col;
        }
    }
}

__global__ void stages_kernel(const int64_t* __restrict__ distinct, int64_t nparts, int32_t B,
                              int64_t* __restrict__ nst) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < nparts; p += (int64_t)gridDim.x * blockDim.x)
        nst[p] = (distinct[p] + B - 1) / B;
}

__global__ void stage_part_kernel(const int64_t* __restrict__ stage_base, int64_t nparts,
                                  int32_t* __restrict__ stage_part) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < nparts; p += (int64_t)gridDim.x * blockDim.x)
        for (int64_t g = stage_base[p]; g < stage_base[p + 1]; ++g) stage_part[g] = (int32_t)p;
}

// per (row, local stage): start of the stage's run inside the row and its length
__global__ void runs_kernel(const int64_t* __restrict__ row_ptr, const uint32_t* __restrict__ rank,
                            const int64_t* __restrict__ stage_base, int64_t nrows, int32_t R, int32_t B,
                            int32_t maxS, int32_t* __restrict__ run_start, int32_t* __restrict__ run_len) {
    const int64_t total = nrows * maxS;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t row = i / maxS;
        const int32_t s = (int32_t)(i % maxS);
        const int64_t p = row / R;
        const int64_t S = stage_base[p + 1] - stage_base[p];
        if (s >= S) { run_start[i] = 0; run_len[i] = 0; continue; }
        const int64_t b = row_ptr[row], e = row_ptr[row + 1];
        auto lower = [&](uint64_t key) {
            int64_t lo = b, hi = e;
            while (lo < hi) {
                const int64_t mid = (lo + hi) >> 1;
                if ((uint64_t)rank[mid] < key) lo = mid + 1; else hi = mid;
            }
            return lo;
        };
        const int64_t s0 = lower((uint64_t)s * B), s1 = lower((uint64_t)(s + 1) * B);
        run_start[i] = (int32_t)(s0 - b);
        run_len[i] = (int32_t)(s1 - s0);
    }
}

// one warp per (global stage, slice): chunks of each lane = ceil(run length / kVec); the block
// stores only the chunks lanes actually have (jagged SELL, plan.h), so its size is kVec * sum.
__global__ void width_kernel(const int32_t* __restrict__ stage_part, const int64_t* __restrict__ stage_base,
                             const int32_t* __restrict__ run_len, int64_t nstages, int32_t SPP, int64_t nrows,
                             int32_t R, int32_t maxS, int64_t* __restrict__ blk_slots,
                             uint16_t* __restrict__ lane_chunks) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x / 32);
    for (int64_t wi = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32; wi < nstages * SPP; wi += warps) {
        const int64_t g = wi / SPP;
        const int32_t w = (int32_t)(wi % SPP);
        const int64_t p = stage_part[g];
        const int64_t s = g - stage_base[p];
        const int64_t row = p * R + (int64_t)w * 32 + lane;
        const int32_t len = (row < nrows) ? run_len[row * maxS + s] : 0;
        const int32_t nch = (len + kVec - 1) / kVec;
        lane_chunks[wi * 32 + lane] = (uint16_t)nch;
        const int32_t tot = __reduce_add_sync(0xffffffffu, nch);
        if (lane == 0) blk_slots[wi] = (int64_t)tot * kVec;
    }
}

// Position of chunk c of `lane` inside its block: chunks are stored chunk-index-major, and within
// chunk c only the lanes that have it, in lane order.  prefix = slots of chunks 0..c-1 / kVec,
// active = lanes having chunk c, rank = active lanes below `lane`.
__device__ __forceinline__ void jagged_pos(const uint16_t* __restrict__ lc, int lane, int64_t c,
                                           int64_t& prefix, int32_t& active, int32_t& rank) {
    prefix = 0;
    active = 0;
    rank = 0;
    for (int l = 0; l < 32; ++l) {
        const int64_t n = lc[l];
        prefix += n < c ? n : c;
        const bool has = n > c;
        active += has;
        rank += (has && l < lane);
    }
}

__global__ void scatter_kernel(const uint32_t* __restrict__ row_ids, const float* __restrict__ vals,
                               const uint32_t* __restrict__ rank, const int64_t* __restrict__ row_ptr,
                               const int32_t* __restrict__ run_start, const int64_t* __restrict__ stage_base,
                               const int64_t* __restrict__ slot_off, const uint16_t* __restrict__ lane_chunks,
                               int64_t nnz, int32_t R, int32_t SPP, int32_t B, int32_t maxS,
                               uint16_t* __restrict__ ind, float* __restrict__ val) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t row = row_ids[e];
        const int64_t p = row / R;
        const int32_t wl = (int32_t)((row % R) >> 5), lane = (int32_t)(row & 31);
        const uint32_t rk = rank[e];
        const int32_t s = (int32_t)(rk / (uint32_t)B);
        const uint32_t local = rk % (uint32_t)B;
        const int64_t j = (e - row_ptr[row]) - run_start[row * maxS + s];
        const int64_t blk = (stage_base[p] + s) * SPP + wl;
        const int64_t base = slot_off[blk];
        const int64_t c = j / kVec, e8 = j % kVec;
        int64_t prefix;
        int32_t active, rnk;
        jagged_pos(lane_chunks + blk * 32, lane, c, prefix, active, rnk);
        const int64_t chunk = base + prefix * kVec;
        ind[chunk + (int64_t)rnk * kVec + e8] = (uint16_t)local;
        val[chunk + (e8 >> 2) * ((int64_t)active * 4) + (int64_t)rnk * 4 + (e8 & 3)] = vals[e];
    }
}

__global__ void gather_u32_f32(const uint32_t* __restrict__ perm, const uint32_t* __restrict__ src_u,
                               const float* __restrict__ src_f, uint32_t* __restrict__ dst_u,
                               float* __restrict__ dst_f, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t q = perm[i];
        dst_u[i] = src_u[q];
        dst_f[i] = src_f[q];
    }
}

template <class T> T read_scalar(const T* dptr, cudaStream_t st) {
    T v{};
    MX_CUDA(cudaMemcpyAsync(&v, dptr, sizeof(T), cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    return v;
}

int bits_for(int64_t n) {
    int b = 1;
    while (b < 32 && ((int64_t)1 << b) < n) ++b;
    return b;
}

}  // namespace

void exclusive_scan_i64(const int64_t* in, int64_t* out, int64_t n, cudaStream_t st) {
    size_t tb = 0;
    MX_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, in, out, n, st));
    DevBuf tmp(tb);
    MX_CUDA(cub::DeviceScan::ExclusiveSum(tmp.get(), tb, in, out, n, st));
    MX_LAUNCHED();
    MX_CUDA(cudaStreamSynchronize(st));
}

void widen_i32_to_i64(const int32_t* in, int64_t* out, int64_t n, cudaStream_t st) {
    if (n == 0) return;
    widen_kernel<<<blocks_for(n), kThreads, 0, st>>>(in, out, n);
    MX_LAUNCHED();
}

void row_ptr_from_sorted(const uint32_t* row_ids, int64_t nnz, int64_t nrows, int64_t* row_ptr, cudaStream_t st) {
    row_ptr_kernel<<<blocks_for(nrows + 1), kThreads, 0, st>>>(row_ids, nnz, nrows, row_ptr);
    MX_LAUNCHED();
}

// stable radix sort of (key, index) pairs: perm_out[i] = original index of the i-th smallest key
void stable_sort_by_key(const uint32_t* keys_in, uint32_t* keys_out, uint32_t* perm_out, int64_t n,
                        int64_t key_range, cudaStream_t st) {
    DevArr<uint32_t> idx;
    idx.alloc(n);
    iota_kernel<<<blocks_for(n), kThreads, 0, st>>>(idx.p(), n);
    MX_LAUNCHED();
    size_t tb = 0;
    const int eb = bits_for(key_range);
    MX_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, keys_in, keys_out, idx.p(), perm_out, n, 0, eb, st));
    DevBuf tmp(tb);
    MX_CUDA(cub::DeviceRadixSort::SortPairs(tmp.get(), tb, keys_in, keys_out, idx.p(), perm_out, n, 0, eb, st));
    MX_LAUNCHED();
    MX_CUDA(cudaStreamSynchronize(st));
}

void build_layout(Layout& L, int64_t nrows, int64_t ncols, int64_t nnz, const uint32_t* row_ids,
                  const uint32_t* cols, const float* vals, int32_t R, int32_t B,
                  const int32_t* in_translate, const int32_t* out_translate, cudaStream_t st) {
    L = Layout{};
    L.nrows = nrows;
    L.ncols = ncols;
    L.nnz = nnz;
    L.R = R;
    L.SPP = R / 32;
    L.B = B;
    L.nparts = ceil_div(nrows, R);
    const int64_t nparts = L.nparts;

    DevArr<int64_t> row_ptr;
    row_ptr.alloc(nrows + 1);
    row_ptr_kernel<<<blocks_for(nrows + 1), kThreads, 0, st>>>(row_ids, nnz, nrows, row_ptr.p());
    MX_LAUNCHED();
    std::vector<int64_t> h_row_ptr(nrows + 1);
    MX_CUDA(cudaMemcpyAsync(h_row_ptr.data(), row_ptr.p(), 8 * (nrows + 1), cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));

    // ---- distinct inputs per partition via chunked bitmaps --------------------------------
    const int64_t words = std::max<int64_t>(1, ceil_div(ncols, 32));
    const int64_t budget = (int64_t)2 << 30;  // bytes for bitmap + word prefix per chunk
    const int64_t chunk = std::max<int64_t>(1, std::min<int64_t>(nparts, budget / (words * 8)));
    const int64_t nchunks = ceil_div(nparts, chunk);
    DevArr<uint32_t> bitmap, wprefix, rank;
    bitmap.alloc(chunk * words);
    wprefix.alloc(chunk * words);
    rank.alloc(nnz);
    DevArr<int64_t> distinct;
    distinct.alloc(nparts);

    auto chunk_entries = [&](int64_t pa, int64_t pb, int64_t& e0, int64_t& e1) {
        e0 = h_row_ptr[std::min<int64_t>(pa * R, nrows)];
        e1 = h_row_ptr[std::min<int64_t>(pb * R, nrows)];
    };
    auto do_bitmap = [&](int64_t pa, int64_t pb) {
        int64_t e0, e1;
        chunk_entries(pa, pb, e0, e1);
        MX_CUDA(cudaMemsetAsync(bitmap.p(), 0, 4 * (pb - pa) * words, st));
        if (e1 > e0) {
            mark_kernel<<<blocks_for(e1 - e0), kThreads, 0, st>>>(row_ids, cols, e0, e1, R, pa, words, bitmap.p());
            MX_LAUNCHED();
        }
        prefix_kernel<<<(unsigned)(pb - pa), kScanThreads, 0, st>>>(bitmap.p(), words, pa, wprefix.p(), distinct.p());
        MX_LAUNCHED();
        if (e1 > e0) {
            rank_kernel<<<blocks_for(e1 - e0), kThreads, 0, st>>>(row_ids, cols, e0, e1, R, pa, words,
                                                                   bitmap.p(), wprefix.p(), rank.p());
            MX_LAUNCHED();
        }
    };
    for (int64_t ci = 0; ci < nchunks; ++ci) do_bitmap(ci * chunk, std::min(nparts, (ci + 1) * chunk));

    // ---- stages and map offsets --------------------------------------------------------------
    DevArr<int64_t> nst, dtmp;
    nst.alloc(nparts + 1);
    dtmp.alloc(nparts + 1);
    MX_CUDA(cudaMemsetAsync(nst.p() + nparts, 0, 8, st));
    stages_kernel<<<blocks_for(nparts), kThreads, 0, st>>>(distinct.p(), nparts, B, nst.p());
    MX_LAUNCHED();
    L.stage_base.alloc(nparts + 1);
    exclusive_scan_i64(nst.p(), L.stage_base.p(), nparts + 1, st);
    MX_CUDA(cudaMemcpyAsync(dtmp.p(), distinct.p(), 8 * nparts, cudaMemcpyDeviceToDevice, st));
    MX_CUDA(cudaMemsetAsync(dtmp.p() + nparts, 0, 8, st));
    L.map_off.alloc(nparts + 1);
    exclusive_scan_i64(dtmp.p(), L.map_off.p(), nparts + 1, st);
    L.nstages = read_scalar(L.stage_base.p() + nparts, st);
    L.nmap = read_scalar(L.map_off.p() + nparts, st);
    {
        std::vector<int64_t> h_nst(nparts);
        MX_CUDA(cudaMemcpyAsync(h_nst.data(), nst.p(), 8 * nparts, cudaMemcpyDeviceToHost, st));
        MX_CUDA(cudaStreamSynchronize(st));
        int64_t mx = 0;
        for (int64_t v : h_nst) mx = std::max(mx, v);
        L.max_stages = (int32_t)std::max<int64_t>(mx, 1);
    }
    const int32_t maxS = L.max_stages;

    // ---- map ------------------------------------------------------------------------------
    L.map.alloc(std::max<int64_t>(L.nmap, 1));
    for (int64_t ci = 0; ci < nchunks; ++ci) {
        const int64_t pa = ci * chunk, pb = std::min(nparts, (ci + 1) * chunk);
        if (nchunks > 1) do_bitmap(pa, pb);  // single chunk: bitmap still holds it
        map_kernel<<<blocks_for((pb - pa) * words), kThreads, 0, st>>>(bitmap.p(), wprefix.p(), words, pb - pa, pa,
                                                                        L.map_off.p(), in_translate, L.map.p());
        MX_LAUNCHED();
    }
    bitmap.reset();
    wprefix.reset();

    // ---- per (row, stage) runs, slice widths, slot offsets ----------------------------------
    DevArr<int32_t> run_start, run_len, stage_part;
    run_start.alloc(nrows * maxS);
    run_len.alloc(nrows * maxS);
    if (nrows > 0) {
        runs_kernel<<<blocks_for(nrows * maxS), kThreads, 0, st>>>(row_ptr.p(), rank.p(), L.stage_base.p(), nrows, R,
                                                                   B, maxS, run_start.p(), run_len.p());
        MX_LAUNCHED();
    }
    stage_part.alloc(std::max<int64_t>(L.nstages, 1));
    stage_part_kernel<<<blocks_for(nparts), kThreads, 0, st>>>(L.stage_base.p(), nparts, stage_part.p());
    MX_LAUNCHED();
    const int64_t nblk = L.nstages * L.SPP;
    DevArr<int64_t> blk_slots;
    blk_slots.alloc(nblk + 1);
    MX_CUDA(cudaMemsetAsync(blk_slots.p(), 0, 8 * (nblk + 1), st));
    L.lane_chunks.alloc(std::max<int64_t>(nblk * 32, 1));
    if (nblk > 0) {
        width_kernel<<<blocks_for(nblk * 32), kThreads, 0, st>>>(stage_part.p(), L.stage_base.p(), run_len.p(),
                                                                 L.nstages, L.SPP, nrows, R, maxS, blk_slots.p(),
                                                                 L.lane_chunks.p());
        MX_LAUNCHED();
    }
    L.slot_off.alloc(nblk + 1);
    exclusive_scan_i64(blk_slots.p(), L.slot_off.p(), nblk + 1, st);
    L.nslots = read_scalar(L.slot_off.p() + nblk, st);
    blk_slots.reset();
    run_len.reset();

    // ---- scatter entries into the slots ---------------------------------------------------
    L.ind.alloc(std::max<int64_t>(L.nslots, 1));
    L.val.alloc(std::max<int64_t>(L.nslots, 1));
    MX_CUDA(cudaMemsetAsync(L.ind.p(), 0, 2 * std::max<int64_t>(L.nslots, 1), st));
    MX_CUDA(cudaMemsetAsync(L.val.p(), 0, 4 * std::max<int64_t>(L.nslots, 1), st));
    if (nnz > 0) {
        scatter_kernel<<<blocks_for(nnz), kThreads, 0, st>>>(row_ids, vals, rank.p(), row_ptr.p(), run_start.p(),
                                                             L.stage_base.p(), L.slot_off.p(), L.lane_chunks.p(), nnz,
                                                             R, L.SPP, B, maxS, L.ind.p(), L.val.p());
        MX_LAUNCHED();
    }
    if (out_translate) {
        L.out_idx.alloc(std::max<int64_t>(nrows, 1));
        MX_CUDA(cudaMemcpyAsync(L.out_idx.p(), out_translate, 4 * nrows, cudaMemcpyDeviceToDevice, st));
    }
    MX_CUDA(cudaStreamSynchronize(st));
}

void build_matrices(Plan& P, cudaStream_t st) {
    // angle tables (reading R1), the same expression as the paper's geometry in DESIGN.md
    std::vector<double> hc(P.m), hs(P.m);
    for (int32_t m = 0; m < P.m; ++m) {
        const double th = (double)m * M_PI / (double)P.m;
        hc[m] = std::cos(th);
        hs[m] = std::sin(th);
    }
    DevArr<double> dc, ds;
    dc.alloc(P.m);
    ds.alloc(P.m);
    MX_CUDA(cudaMemcpyAsync(dc.p(), hc.data(), 8 * P.m, cudaMemcpyHostToDevice, st));
    MX_CUDA(cudaMemcpyAsync(ds.p(), hs.data(), 8 * P.m, cudaMemcpyHostToDevice, st));
    Geometry G;
    G.cos_t = dc.p();
    G.sin_t = ds.p();

    // a3: this rank's tomogram and sinogram subdomains (whole domains at P = 1)
    decompose(P, G, st);
    const int64_t npix = P.t1 - P.t0;

    // 1. rows of A_p = footprint rays (every ray at P = 1), count pass + scan
    DevArr<int32_t> row_len;
    const int64_t nrows = P.nfp = footprint(P, G, row_len, st);
    DevArr<int64_t> len64, row_ptr;
    len64.alloc(nrows + 1);
    row_ptr.alloc(nrows + 1);
    widen_i32_to_i64(row_len.p(), len64.p(), nrows, st);
    MX_CUDA(cudaMemsetAsync(len64.p() + nrows, 0, 8, st));
    exclusive_scan_i64(len64.p(), row_ptr.p(), nrows + 1, st);
    len64.reset();
    row_len.reset();
    const int64_t nnz = read_scalar(row_ptr.p() + nrows, st);
    if (nnz >= ((int64_t)1 << 32))
        fail(MEMXCT_ERR_UNSUPPORTED, "nnz >= 2^32 on one GPU; shard the problem over more GPUs");

    // 2. emit (local Hilbert pixel, length, row) for the segments inside this rank's pixels
    DevArr<uint32_t> a_col, a_row;
    DevArr<float> a_val;
    a_col.alloc(nnz);
    a_row.alloc(nnz);
    a_val.alloc(nnz);
    trace_emit(P, G, P.nranks == 1 ? nullptr : P.fp_rays.p(), nrows, P.t0, P.t1, row_ptr.p(), a_col.p(),
               a_val.p(), a_row.p(), st);
    row_ptr.reset();

    const bool natural = (P.opt.vector_order == 0);  // P = 1 only
    const int32_t R = P.part_rows;
    const int32_t B = P.opt.precision == 1 ? P.buffer_entries / 2 : P.buffer_entries;

    // 3. A_p^T: stable sort by pixel (order-preserving transposition)
    DevArr<uint32_t> t_row, t_col, perm;
    DevArr<float> t_val;
    t_row.alloc(nnz);
    perm.alloc(nnz);
    stable_sort_by_key(a_col.p(), t_row.p(), perm.p(), nnz, std::max<int64_t>(npix, 1), st);
    a_col.reset();
    t_col.alloc(nnz);
    t_val.alloc(nnz);
    gather_u32_f32<<<blocks_for(nnz), kThreads, 0, st>>>(perm.p(), a_row.p(), a_val.p(), t_col.p(), t_val.p(), nnz);
    MX_LAUNCHED();
    MX_CUDA(cudaStreamSynchronize(st));
    a_row.reset();
    a_val.reset();
    perm.reset();
    build_layout(P.back, npix, nrows, nnz, t_row.p(), t_col.p(), t_val.p(), R, B,
                 natural ? P.sino_nat_of_h.p() : nullptr, natural ? P.tomo_nat_of_h.p() : nullptr, st);

    // 4. A_p with ascending pixels inside each row: stable sort of the A_p^T entries by row
    DevArr<uint32_t> f_row, f_col;
    DevArr<float> f_val;
    f_row.alloc(nnz);
    perm.alloc(nnz);
    stable_sort_by_key(t_col.p(), f_row.p(), perm.p(), nnz, std::max<int64_t>(nrows, 1), st);
    t_col.reset();
    f_col.alloc(nnz);
    f_val.alloc(nnz);
    gather_u32_f32<<<blocks_for(nnz), kThreads, 0, st>>>(perm.p(), t_row.p(), t_val.p(), f_col.p(), f_val.p(), nnz);
    MX_LAUNCHED();
    MX_CUDA(cudaStreamSynchronize(st));
    t_row.reset();
    t_val.reset();
    perm.reset();
    build_layout(P.fwd, nrows, npix, nnz, f_row.p(), f_col.p(), f_val.p(), R, B,
                 natural ? P.tomo_nat_of_h.p() : nullptr, natural ? P.sino_nat_of_h.p() : nullptr, st);

    // a6: exchange maps of the sparse all-to-allv (P > 1)
    build_exchange(P, st);
}

}  // namespace mx
