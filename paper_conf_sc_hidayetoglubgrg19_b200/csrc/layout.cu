// layout.cu -- preprocessing: Siddon-traced A_p, its order-preserving transposition,
// and the multi-stage buffered layout of both directions, all on the device, built
// in CHUNKS of whole partitions so the temporaries stay within a memory budget (configs 4-5
// exceed 2^32 nonzeros per direction; the finished layouts alone take most of the 180 GB).
//
// Per direction, rows are generated chunk by chunk, sorted by (row, input):
//   A   (rows = footprint rays):   emit the chunk's rays (trace.cu), then a segmented sort of
//                                  every ray's entries by pixel;
//   A^T (rows = local pixels):     re-trace the footprint rays with a pixel-range filter for the
//                                  chunk's pixels, then a STABLE radix sort on the pixel key --
//                                  entries of a pixel keep ascending ray order: the scan-based,
//                                  order-preserving transposition of P:847-858 (no atomics).
// Two passes over the chunks: pass 1 sizes everything (distinct inputs, stages and slots per
// partition), the exact final arrays are allocated, pass 2 regenerates the chunk (unless there
// is only one, which is kept) and scatters it.
//
// Layout per partition p = R consecutive rows (one CTA), readings R10/R11:
//   * distinct inputs of p by a per-partition bitmap over the input domain; a popcount prefix
//     gives every entry the rank of its input among them, in ascending Hilbert order (the stage
//     map order);
//   * stage s = ranks [s*B, (s+1)*B): map[s*B + i] = input index, 16-bit local index
//     i = rank % B;
//   * per (stage, 32-row slice) block: jagged SELL-32 (plan.h): each lane's run rounded up to
//     kVec slots, chunk c stored only for the lanes that have it.
#include <cub/block/block_scan.cuh>
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_segmented_sort.cuh>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <functional>
#include <vector>

#include "plan.h"

namespace mx {

namespace {

constexpr int kThreads = 256;

inline unsigned blocks_for(int64_t n, int threads = kThreads) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, threads), 1 << 30));
}

#define MX_LOOP(i, n) for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < (n); i += (int64_t)gridDim.x * blockDim.x)

template <class T> __global__ void iota_kernel(T* out, int64_t n) { MX_LOOP(i, n) out[i] = (T)i; }

__global__ void widen_kernel(const int32_t* in, int64_t* out, int64_t n) { MX_LOOP(i, n) out[i] = in[i]; }

// row_ptr[r] = first entry with row_ids >= r0 + r (row_ids sorted ascending), r in [0, nrows]
__global__ void row_ptr_kernel(const uint32_t* __restrict__ row_ids, int64_t nnz, int64_t r0, int64_t nrows,
                               int64_t* __restrict__ row_ptr) {
    MX_LOOP(r, nrows + 1) {
        int64_t lo = 0, hi = nnz;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if ((int64_t)row_ids[mid] < r0 + r) lo = mid + 1; else hi = mid;
        }
        row_ptr[r] = lo;
    }
}

// mark the input of every entry of partitions [pa, ...) in the sub-chunk bitmap
__global__ void mark_kernel(const uint32_t* __restrict__ row_ids, const uint32_t* __restrict__ cols,
                            int64_t e0, int64_t e1, const int32_t* __restrict__ row_part, int64_t pa, int64_t words,
                            uint32_t* __restrict__ bitmap) {
    for (int64_t e = e0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < e1; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t p = row_part[row_ids[e]] - pa;
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
                            int64_t e0, int64_t e1, const int32_t* __restrict__ row_part, int64_t pa, int64_t words,
                            const uint32_t* __restrict__ bitmap, const uint32_t* __restrict__ word_prefix,
                            uint32_t* __restrict__ rank) {
    for (int64_t e = e0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < e1; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t p = row_part[row_ids[e]] - pa;
        const uint32_t c = cols[e];
        const int64_t w = p * words + (c >> 5);
        rank[e] = word_prefix[w] + (uint32_t)__popc(bitmap[w] & ((1u << (c & 31)) - 1u));
    }
}

// map[map_off[p] + rank] = translated input of every set bit of partition p's bitmap
// (slab stage order: the bitmap is over the partition's class order col' = K_c[col]; inv holds
// the C inverse orders [C][ncols] and part_class the class of every partition)
__global__ void map_kernel(const uint32_t* __restrict__ bitmap, const uint32_t* __restrict__ word_prefix,
                           int64_t words, int64_t nsub, int64_t pa, const int64_t* __restrict__ map_off,
                           const int32_t* __restrict__ translate, const int32_t* __restrict__ inv,
                           const int32_t* __restrict__ part_class, int64_t ncols, int32_t* __restrict__ map) {
    MX_LOOP(i, nsub * words) {
        uint32_t b = bitmap[i];
        if (!b) continue;
        const int64_t p = i / words, w = i % words;
        int64_t r = map_off[pa + p] + word_prefix[i];
        const int32_t* iv = inv ? inv + (int64_t)part_class[pa + p] * ncols : nullptr;
        while (b) {
            const int bit = __ffs(b) - 1;
            b &= b - 1;
            int64_t col = w * 32 + bit;
            if (iv) col = iv[col];
            map[r++] = translate ? translate[col] : (int32_t)col;
        }
    }
}

__global__ void stages_kernel(const int64_t* __restrict__ distinct, int64_t n, int32_t B, int64_t* __restrict__ nst) {
    MX_LOOP(p, n) nst[p] = (distinct[p] + B - 1) / B;
}

__global__ void stage_part_kernel(const int64_t* __restrict__ stage_base, int64_t nparts,
                                  int32_t* __restrict__ stage_part) {
    MX_LOOP(p, nparts)
    for (int64_t g = stage_base[p]; g < stage_base[p + 1]; ++g) stage_part[g] = (int32_t)p;
}

// per (chunk row, local stage): start of the stage's run inside the row and its length
__global__ void runs_kernel(const int64_t* __restrict__ row_ptr, const uint32_t* __restrict__ rank,
                            const int64_t* __restrict__ nst, int64_t ra, int64_t nr,
                            const int32_t* __restrict__ row_part, int32_t B, int32_t maxS,
                            int32_t* __restrict__ run_start, int32_t* __restrict__ run_len) {
    MX_LOOP(i, nr * maxS) {
        const int64_t r = i / maxS;
        const int32_t s = (int32_t)(i % maxS);
        const int64_t S = nst[row_part[ra + r]];
        if (s >= S) { run_start[i] = 0; run_len[i] = 0; continue; }
        const int64_t b = row_ptr[r], e = row_ptr[r + 1];
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

// one warp per chunk block (local stage, slice): chunks of each lane = ceil(run / kVec); the
// block stores only the chunks lanes actually have (jagged SELL, plan.h)
__global__ void width_kernel(const int32_t* __restrict__ stage_part, const int64_t* __restrict__ cs_base,
                             const int32_t* __restrict__ run_len, int64_t nblk, int32_t SPP, int64_t pa,
                             int64_t ra, const int64_t* __restrict__ prow0, int32_t maxS,
                             int64_t* __restrict__ blk_slots, uint16_t* __restrict__ lane_chunks) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x / 32);
    for (int64_t wi = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32; wi < nblk; wi += warps) {
        const int64_t g = wi / SPP;
        const int32_t w = (int32_t)(wi % SPP);
        const int64_t pl = stage_part[g];
        const int64_t s = g - cs_base[pl];
        const int64_t row = prow0[pa + pl] + (int64_t)w * 32 + lane;
        const int32_t len = (row < prow0[pa + pl + 1]) ? run_len[(row - ra) * maxS + s] : 0;
        const int32_t nch = (len + kVec - 1) / kVec;
        lane_chunks[wi * 32 + lane] = (uint16_t)nch;
        const int32_t tot = __reduce_add_sync(0xffffffffu, nch);
        if (lane == 0) blk_slots[wi] = (int64_t)tot * kVec;
    }
}

// Bank-aware order inside the (row, stage) runs (FP32 plans tuned for K >= 2 slices, where the
// shared-memory gather of K-wide entries, not HBM, limits the SpMM).  A K-wide entry at local
// index i sits in bank group i mod C (C = 8 groups for 16 B entries, 16 for 8 B), and a warp's
// gather is served in phases of C lanes; the slots of the C lanes of a phase at one position j
// should hit distinct groups.
// Step 1 (this kernel, one warp per run): stable counting sort of the run by bank class; writes
// srt[b + p] = offset (inside the run) of the p-th entry in (class, local index) order.
__global__ void bank_order_kernel(const uint32_t* __restrict__ rank, const int64_t* __restrict__ row_ptr,
                                  const int32_t* __restrict__ run_start, const int32_t* __restrict__ run_len,
                                  int64_t nr, int32_t maxS, int64_t ra, int32_t B, int32_t C,
                                  int32_t* __restrict__ srt) {
    const int lane = threadIdx.x & 31;
    const unsigned lt = (1u << lane) - 1u;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x / 32);
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32; i < nr * maxS; i += warps) {
        const int32_t len = run_len[i];
        if (len == 0) continue;
        const int64_t r = i / maxS;
        const int64_t b = row_ptr[r] + run_start[i];
        // class counts: lane c holds count of class c
        int32_t cnt = 0;
        for (int32_t k0 = 0; k0 < len; k0 += 32) {
            const int32_t k = k0 + lane;
            const int32_t cls = k < len ? (int32_t)((rank[b + k] % (uint32_t)B) & (C - 1)) : 32;
            for (int32_t c = 0; c < C; ++c) {
                const unsigned m = __ballot_sync(0xffffffffu, cls == c);
                if (lane == c) cnt += __popc(m);
            }
        }
        // exclusive scan over classes -> base of each class; running offset per class
        int32_t incl = cnt;
        for (int o = 1; o < 32; o <<= 1) {
            const int32_t v = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += v;
        }
        int32_t next = incl - cnt;  // lane c: next free position of class c
        for (int32_t k0 = 0; k0 < len; k0 += 32) {
            const int32_t k = k0 + lane;
            const bool valid = k < len;
            const int32_t cls = valid ? (int32_t)((rank[b + k] % (uint32_t)B) & (C - 1)) : 32;
            const unsigned same = __match_any_sync(0xffffffffu, cls);
            const int32_t pos = __shfl_sync(0xffffffffu, next, cls & 31) + __popc(same & lt);
            if (valid) srt[b + pos] = k;
            for (int32_t c = 0; c < C; ++c) {
                const unsigned m = __ballot_sync(0xffffffffu, cls == c);
                if (lane == c) next += __popc(m);
            }
        }
    }
}

// Step 2 (one thread per (group of C lanes, stage)): greedy schedule.  At every slot position j,
// lanes in order take, from their remaining entries, the class not yet used at j with the most
// entries left (else the fullest class: a conflict); inside a class, ascending local index.
// jnew[e] = position of entry e inside its run.  Simulated on random runs of cfg3 size: 1.09
// wavefronts per phase vs 2.47 for ascending order.
constexpr int kMaxC = 16;
__global__ void bank_greedy_kernel(const uint32_t* __restrict__ rank, const int64_t* __restrict__ row_ptr,
                                   const int32_t* __restrict__ run_start, const int32_t* __restrict__ run_len,
                                   const int32_t* __restrict__ srt, int64_t nr, int32_t maxS, int32_t B, int32_t C,
                                   int32_t* __restrict__ jnew) {
    const int64_t ngroups = (nr + C - 1) / C;
    MX_LOOP(t, ngroups * maxS) {
        const int64_t g = t / maxS;
        const int32_t s = (int32_t)(t % maxS);
        int32_t cnt[kMaxC][kMaxC], nxt[kMaxC][kMaxC], len[kMaxC];
        int64_t base[kMaxC];
        int32_t maxlen = 0;
        for (int32_t i = 0; i < C; ++i) {
            const int64_t r = g * C + i;
            len[i] = 0;
            base[i] = 0;
            for (int32_t c = 0; c < C; ++c) cnt[i][c] = 0;
            if (r >= nr) continue;
            const int64_t ri = r * maxS + s;
            len[i] = run_len[ri];
            base[i] = row_ptr[r] + run_start[ri];
            for (int32_t k = 0; k < len[i]; ++k) ++cnt[i][(rank[base[i] + k] % (uint32_t)B) & (C - 1)];
            int32_t acc = 0;
            for (int32_t c = 0; c < C; ++c) { nxt[i][c] = acc; acc += cnt[i][c]; }
            maxlen = max(maxlen, len[i]);
        }
        for (int32_t j = 0; j < maxlen; ++j) {
            uint32_t used = 0;
            for (int32_t i = 0; i < C; ++i) {
                if (j >= len[i]) continue;
                int32_t best = -1, bestn = 0, fb = 0, fbn = 0;
                for (int32_t c = 0; c < C; ++c) {
                    const int32_t n = cnt[i][c];
                    if (n > bestn && !((used >> c) & 1u)) { best = c; bestn = n; }
                    if (n > fbn) { fb = c; fbn = n; }
                }
                const int32_t c = best >= 0 ? best : fb;
                used |= 1u << c;
                const int32_t k = srt[base[i] + nxt[i][c]];
                jnew[base[i] + k] = j;
                ++nxt[i][c];
                --cnt[i][c];
            }
        }
    }
}

// pass 1: slots of every partition of the chunk
__global__ void part_slots_kernel(const int64_t* __restrict__ blk_slots, const int64_t* __restrict__ cs_base,
                                  int64_t np, int32_t SPP, int64_t pa, int64_t* __restrict__ slots_p) {
    MX_LOOP(p, np) {
        int64_t s = 0;
        for (int64_t b = cs_base[p] * SPP; b < cs_base[p + 1] * SPP; ++b) s += blk_slots[b];
        slots_p[pa + p] = s;
    }
}

__global__ void add_offset_kernel(const int64_t* __restrict__ in, int64_t n, int64_t off, int64_t* __restrict__ out) {
    MX_LOOP(i, n) out[i] = in[i] + off;
}

// Position of chunk c of `lane` inside its block: chunks are stored chunk-index-major, and within
// chunk c only the lanes that have it, in lane order.  prefix = chunks stored before chunk c,
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
                               const int32_t* __restrict__ jnew, int64_t nnz, int64_t ra,
                               const int32_t* __restrict__ row_part, const int64_t* __restrict__ prow0, int32_t SPP,
                               int32_t B, int32_t maxS, uint16_t* __restrict__ ind, float* __restrict__ val) {
    MX_LOOP(e, nnz) {
        const int64_t row = row_ids[e];
        const int64_t r = row - ra;
        const int64_t p = row_part[row];
        const int64_t lr = row - prow0[p];  // row inside its partition: warp lr / 32, lane lr % 32
        const int32_t wl = (int32_t)(lr >> 5), lane = (int32_t)(lr & 31);
        const uint32_t rk = rank[e];
        const int32_t s = (int32_t)(rk / (uint32_t)B);
        const uint32_t local = rk % (uint32_t)B;
        const int64_t j = jnew ? (int64_t)jnew[e] : (e - row_ptr[r]) - run_start[r * maxS + s];
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
    MX_LOOP(i, n) {
        const uint32_t q = perm[i];
        dst_u[i] = src_u[q];
        dst_f[i] = src_f[q];
    }
}

__global__ void offset_u32_kernel(uint32_t* v, int64_t n, uint32_t add) { MX_LOOP(i, n) v[i] += add; }

// row_part[r] = partition of row r
__global__ void row_part_kernel(const int64_t* __restrict__ prow0, int64_t np, int32_t* __restrict__ row_part) {
    MX_LOOP(p, np)
    for (int64_t r = prow0[p]; r < prow0[p + 1]; ++r) row_part[r] = (int32_t)p;
}

template <class T> T read_scalar(const T* dptr, cudaStream_t st) {
    T v{};
    MX_CUDA(cudaMemcpyAsync(&v, dptr, sizeof(T), cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    return v;
}

template <class T> std::vector<T> to_host(const T* d, int64_t n, cudaStream_t st) {
    std::vector<T> h(std::max<int64_t>(n, 0));
    if (n > 0) MX_CUDA(cudaMemcpyAsync(h.data(), d, sizeof(T) * n, cudaMemcpyDeviceToHost, st));
    MX_CUDA(cudaStreamSynchronize(st));
    return h;
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
    row_ptr_kernel<<<blocks_for(nrows + 1), kThreads, 0, st>>>(row_ids, nnz, 0, nrows, row_ptr);
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

// ---- chunked layout builder ------------------------------------------------------------------
namespace {

struct Partitions {         // host: partition p = rows [row0[p], row0[p+1]), nnz[p] nonzeros
    std::vector<int64_t> row0, nnz;
    bool balanced = false;
};

struct Entries {            // one chunk of a direction, sorted by (row, input)
    DevArr<uint32_t> row;   // absolute row ids
    DevArr<uint32_t> col;   // input index (plan order, local to the rank)
    DevArr<float> val;
    int64_t n = 0;
    void reset() { row.reset(); col.reset(); val.reset(); n = 0; }
};
using Generator = std::function<void(int64_t ra, int64_t rb, Entries& out, cudaStream_t st)>;

struct Builder {
    Layout& L;
    int64_t nrows, ncols;
    int32_t R, B, SPP;
    const int32_t* in_translate;
    const int32_t* row_part;        // device: partition of every row
    const int64_t* prow0;           // device: first row of every partition (nparts + 1)
    std::vector<int64_t> h_prow0;   // host copy
    int64_t words;
    int64_t bitmap_parts;   // partitions per bitmap sub-chunk
    int32_t bank_classes;   // 0 = ascending local index in every run; else bank-aware order
    const int32_t* col_inv = nullptr;     // slab stage order: [C][ncols] col' -> col (else null)
    const int32_t* part_class = nullptr;  // slab stage order: class of every partition
    DevArr<int64_t> distinct, nst, slots_p;
    std::vector<int64_t> h_stage_base, h_part_slot;

    // ranks of one chunk's entries (and, in pass 2, the stage maps)
    void ranks(const Entries& E, int64_t pa, int64_t pb, const std::vector<int64_t>& h_row_ptr, int64_t ra,
               DevArr<uint32_t>& rank, bool write_map, cudaStream_t st) {
        DevArr<uint32_t> bitmap, wprefix;
        const int64_t q = std::min<int64_t>(bitmap_parts, pb - pa);
        bitmap.alloc(q * words);
        wprefix.alloc(q * words);
        for (int64_t qa = pa; qa < pb; qa += q) {
            const int64_t qb = std::min(pb, qa + q);
            const int64_t e0 = h_row_ptr[h_prow0[qa] - ra];
            const int64_t e1 = h_row_ptr[h_prow0[qb] - ra];
            MX_CUDA(cudaMemsetAsync(bitmap.p(), 0, 4 * (qb - qa) * words, st));
            if (e1 > e0) {
                mark_kernel<<<blocks_for(e1 - e0), kThreads, 0, st>>>(E.row.p(), E.col.p(), e0, e1, row_part, qa, words,
                                                                      bitmap.p());
                MX_LAUNCHED();
            }
            prefix_kernel<<<(unsigned)(qb - qa), kScanThreads, 0, st>>>(bitmap.p(), words, qa, wprefix.p(),
                                                                        distinct.p());
            MX_LAUNCHED();
            if (e1 > e0) {
                rank_kernel<<<blocks_for(e1 - e0), kThreads, 0, st>>>(E.row.p(), E.col.p(), e0, e1, row_part, qa, words,
                                                                      bitmap.p(), wprefix.p(), rank.p());
                MX_LAUNCHED();
            }
            if (write_map) {
                map_kernel<<<blocks_for((qb - qa) * words), kThreads, 0, st>>>(bitmap.p(), wprefix.p(), words,
                                                                                qb - qa, qa, L.map_off.p(),
                                                                                in_translate, col_inv, part_class,
                                                                                ncols, L.map.p());
                MX_LAUNCHED();
            }
        }
    }

    void process(const Entries& E, int64_t pa, int64_t pb, int pass, cudaStream_t st) {
        const int64_t ra = h_prow0[pa], rb = h_prow0[pb], nr = rb - ra, np = pb - pa;
        DevArr<int64_t> row_ptr;
        row_ptr.alloc(nr + 1);
        row_ptr_kernel<<<blocks_for(nr + 1), kThreads, 0, st>>>(E.row.p(), E.n, ra, nr, row_ptr.p());
        MX_LAUNCHED();
        const auto h_row_ptr = to_host(row_ptr.p(), nr + 1, st);
        DevArr<uint32_t> rank;
        rank.alloc(std::max<int64_t>(E.n, 1));
        ranks(E, pa, pb, h_row_ptr, ra, rank, pass == 2, st);
        stages_kernel<<<blocks_for(np), kThreads, 0, st>>>(distinct.p() + pa, np, B, nst.p() + pa);
        MX_LAUNCHED();
        const auto h_nst = to_host(nst.p() + pa, np, st);
        int64_t maxS = 1;
        std::vector<int64_t> h_cs(np + 1, 0);
        for (int64_t p = 0; p < np; ++p) {
            maxS = std::max(maxS, h_nst[p]);
            h_cs[p + 1] = h_cs[p] + h_nst[p];
        }
        const int64_t ns = h_cs[np], nblk = ns * SPP;
        DevArr<int64_t> cs;
        cs.alloc(np + 1);
        MX_CUDA(cudaMemcpyAsync(cs.p(), h_cs.data(), 8 * (np + 1), cudaMemcpyHostToDevice, st));
        DevArr<int32_t> run_start, run_len, stage_part;
        run_start.alloc(std::max<int64_t>(nr * maxS, 1));
        run_len.alloc(std::max<int64_t>(nr * maxS, 1));
        if (nr > 0) {
            runs_kernel<<<blocks_for(nr * maxS), kThreads, 0, st>>>(row_ptr.p(), rank.p(), nst.p(), ra, nr, row_part,
                                                                    B, (int32_t)maxS, run_start.p(), run_len.p());
            MX_LAUNCHED();
        }
        stage_part.alloc(std::max<int64_t>(ns, 1));
        stage_part_kernel<<<blocks_for(np), kThreads, 0, st>>>(cs.p(), np, stage_part.p());
        MX_LAUNCHED();
        DevArr<int64_t> blk_slots;
        DevArr<uint16_t> lanes;
        blk_slots.alloc(nblk + 1);
        MX_CUDA(cudaMemsetAsync(blk_slots.p(), 0, 8 * (nblk + 1), st));
        // pass 2 writes the lane counts straight into the final array
        uint16_t* lane_out = nullptr;
        if (pass == 2) lane_out = L.lane_chunks.p() + h_stage_base[pa] * SPP * 32;
        else { lanes.alloc(std::max<int64_t>(nblk * 32, 1)); lane_out = lanes.p(); }
        if (nblk > 0) {
            width_kernel<<<blocks_for(nblk * 32), kThreads, 0, st>>>(stage_part.p(), cs.p(), run_len.p(), nblk, SPP,
                                                                     pa, ra, prow0, (int32_t)maxS, blk_slots.p(),
                                                                     lane_out);
            MX_LAUNCHED();
        }
        DevArr<int32_t> jnew;
        if (pass == 2 && bank_classes > 0 && E.n > 0 && nr > 0) {
            DevArr<int32_t> srt;
            srt.alloc(E.n);
            jnew.alloc(E.n);
            bank_order_kernel<<<blocks_for(nr * maxS * 32), kThreads, 0, st>>>(rank.p(), row_ptr.p(), run_start.p(),
                                                                              run_len.p(), nr, (int32_t)maxS, ra, B,
                                                                              bank_classes, srt.p());
            MX_LAUNCHED();
            bank_greedy_kernel<<<blocks_for(ceil_div(nr, bank_classes) * maxS, 128), 128, 0, st>>>(
                rank.p(), row_ptr.p(), run_start.p(), run_len.p(), srt.p(), nr, (int32_t)maxS, B, bank_classes,
                jnew.p());
            MX_LAUNCHED();
            MX_CUDA(cudaStreamSynchronize(st));
        }
        run_len.reset();
        if (pass == 1) {
            part_slots_kernel<<<blocks_for(np), kThreads, 0, st>>>(blk_slots.p(), cs.p(), np, SPP, pa, slots_p.p());
            MX_LAUNCHED();
            MX_CUDA(cudaStreamSynchronize(st));
            return;
        }
        // pass 2: block offsets = partition slot base + scan of the chunk's block sizes
        DevArr<int64_t> boff;
        boff.alloc(nblk + 1);
        exclusive_scan_i64(blk_slots.p(), boff.p(), nblk + 1, st);
        if (nblk > 0) {
            add_offset_kernel<<<blocks_for(nblk), kThreads, 0, st>>>(boff.p(), nblk, h_part_slot[pa],
                                                                     L.slot_off.p() + h_stage_base[pa] * SPP);
            MX_LAUNCHED();
        }
        if (E.n > 0) {
            scatter_kernel<<<blocks_for(E.n), kThreads, 0, st>>>(E.row.p(), E.val.p(), rank.p(), row_ptr.p(),
                                                                 run_start.p(), L.stage_base.p(), L.slot_off.p(),
                                                                 L.lane_chunks.p(), jnew.p(), E.n, ra, row_part, prow0,
                                                                 SPP, B, (int32_t)maxS, L.ind.p(), L.val.p());
            MX_LAUNCHED();
        }
        MX_CUDA(cudaStreamSynchronize(st));
    }
};

// Launch order of the partitions (MEMXCT_PART_ORDER: 0 = partition order (default), 1 = heaviest
// first).  A CTA's time is ~ its streamed bytes (6 B per slot, 8 B per map entry, 4 B per row)
// plus a gather round trip per stage; longest-processing-time order leaves the lightest
// partitions for the last, partly filled wave.  Measured on one B200 (profiles/r01h_order_ab.jsonl):
// cfg3 back -1.6 %, forward +1.1 %, cfg2 and cfg4 +0.5-1 % -- within a wave-tail effect of ~1 %,
// so partition (Hilbert) order stays the default.
void set_part_order(Layout& L, const std::vector<int64_t>& row0, const std::vector<int64_t>& part_slot,
                    const std::vector<int64_t>& stage_base, cudaStream_t st) {
    int mode = 0;
    if (const char* e = std::getenv("MEMXCT_PART_ORDER")) mode = atoi(e);
    const int64_t np = L.nparts;
    if (mode == 0 || np < 2) return;
    constexpr int64_t kStageCost = 16384;  // bytes of streaming time per stage barrier + gather
    const auto moff = to_host(L.map_off.p(), np + 1, st);
    std::vector<int64_t> work(np);
    for (int64_t p = 0; p < np; ++p)
        work[p] = 6 * (part_slot[p + 1] - part_slot[p]) + 8 * (moff[p + 1] - moff[p]) +
                  4 * (row0[p + 1] - row0[p]) + kStageCost * (stage_base[p + 1] - stage_base[p]);
    std::vector<int32_t> ord(np);
    for (int64_t p = 0; p < np; ++p) ord[p] = (int32_t)p;
    std::stable_sort(ord.begin(), ord.end(), [&](int32_t u, int32_t v) { return work[u] > work[v]; });
    L.part_order.alloc(np);
    MX_CUDA(cudaMemcpyAsync(L.part_order.p(), ord.data(), 4 * np, cudaMemcpyHostToDevice, st));
    MX_CUDA(cudaStreamSynchronize(st));  // ord is a host temporary
}

// budget of chunk entries: what is free after the finished layouts of both directions
// Default tuning of one direction with `rows` output rows on this rank (B200 sweeps:
// profiles/r01_sweep.md, r01_sweep_cfg2.md, r01_sweep_spmm.md, r01_virtual_scaling.md).
//  * R (rows per partition = threads per CTA, a multiple of 32): 1024 (32 warps, one CTA per SM;
//    Hilbert-aligned partitions, the best input reuse) whenever that gives >= 0.8 CTAs per SM --
//    ~120 streaming SMs already saturate HBM (virtual-rank sweep: cfg3 A^T at P = 8, 128 CTAs,
//    is as fast as any balanced split).  Smaller problems would leave most SMs idle: then R is
//    the largest multiple of 32 in [128, 1024] whose parts spread over the SMs with
//    w / ceil(w) >= 0.97, w = parts / SMs (else the most balanced one); cfg2: 640 / 448, 4.5 %
//    more CG iter/s than 256.
//  * B (stage buffer entries): 36 fp32 entries per row for one slice (144 KB at R = 1024); for
//    k-slice plans 192 KB of k-wide entries (a 200 KB buffer leaves 28 KB of L1 for the gathers).
// Drifting stages (spmv_f32_drift_kernel): MEMXCT_DRIFT=1 selects it, MEMXCT_DRIFT_B sets its
// auto stage size (3 buffers of B entries share the CTA's shared memory).
static bool drift_requested() {
    const char* e = std::getenv("MEMXCT_DRIFT");
    return e && atoi(e) != 0;
}
// Three buffers of 13312 entries (156 KB) are the largest that keep the shared-memory carve-out
// at 164 KB and so 92 KB of L1 for the stream's loads in flight; 16384 (192 KB) selects the 196 KB
// carve-out and leaves 60 KB.  Config-5 shard forward (asynchronous gather): 7.54 ms at 16384,
// 7.42 at 13312, 7.48 at 12288 although the smaller stages raise the slab padding 3.8 -> 4.7 %
// (r02aw, profiles/r02aw_drift_b_cfg5.jsonl; with the synchronous gather 16384 was best, r01i).
static int32_t drift_auto_b() {
    const char* e = std::getenv("MEMXCT_DRIFT_B");
    return e ? std::max(256, atoi(e)) : 13312;
}

void resolve_tuning(const Plan& P, int64_t rows, int32_t* R_out, int32_t* B_out) {
    int dev = 0, sms = 148;
    MX_CUDA(cudaGetDevice(&dev));
    MX_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    int32_t R = (int32_t)P.opt.part_rows;
    if (R == 0 && 5 * ceil_div(std::max<int64_t>(rows, 1), (int64_t)1024) >= 4 * (int64_t)sms) R = 1024;
    if (R == 0) {
        rows = std::max<int64_t>(rows, 1);
        double best = -1.0;
        int32_t best_r = 128;
        for (int32_t cand = 1024; cand >= 128; cand -= 32) {
            const double w = (double)ceil_div(rows, (int64_t)cand) / sms;
            const double eff = w / std::ceil(w);
            if (eff >= 0.97) { best_r = cand; break; }
            if (eff > best + 1e-12) { best = eff; best_r = cand; }
        }
        R = best_r;
    }
    int32_t B = (int32_t)P.opt.buffer_entries;
    if (B == 0) {
        int32_t k = 1;
        while (k < P.opt.slices) k *= 2;  // batched calls stage k slices per buffer entry
        // k >= 2: 192 KB of fp32 slice groups at k >= 4; k = 2 stages as many entries as k = 4
        // (96 KB): cfg3 K = 2 SpMM 1.742 ms at B = 12288 vs 1.795 at 24576, and every size
        // above 192 KB falls off a cliff (K = 4 at 14336: 2.49 ms), profiles/r01n_spmm_bigB.jsonl
        B = (k == 1) ? std::min<int32_t>(drift_requested() ? drift_auto_b() : 57344, 36 * R)
                     : std::min<int32_t>(49152, 144 * R) / std::max<int32_t>(k, 4);
        B = std::max<int32_t>(256, B - B % 256);
    }
    *R_out = R;
    *B_out = B;
}

int64_t chunk_budget(int64_t nnz_both_dirs_remaining) {
    size_t fr = 0, tot = 0;
    MX_CUDA(cudaMemGetInfo(&fr, &tot));
    const double reserve = 6.3 * (double)nnz_both_dirs_remaining + 3e9;
    const double avail = (double)fr - reserve;
    const int64_t cap = ((int64_t)1 << 31) - 1;  // CUB segmented sort: int item counts
    if (const char* e = std::getenv("MEMXCT_BUILD_CHUNK")) return std::max<int64_t>(1, std::min<int64_t>(cap, atoll(e)));
    return std::max<int64_t>(1 << 24, std::min<int64_t>(cap, (int64_t)(avail / 48.0)));
}

void build_direction(Layout& L, int64_t nrows, int64_t ncols, const Partitions& parts, int32_t R,
                     int32_t B, const Generator& gen, const int32_t* in_translate, const int32_t* out_translate,
                     int64_t budget, int32_t bank_classes, cudaStream_t st, const int32_t* col_inv = nullptr,
                     const int32_t* part_class = nullptr) {
    L = Layout{};
    L.nrows = nrows;
    L.ncols = ncols;
    L.R = R;
    L.SPP = R / 32;
    L.B = B;
    L.nparts = (int64_t)parts.row0.size() - 1;
    L.balanced = parts.balanced;
    L.drift = drift_requested() && 12 * (int64_t)B <= 224 * 1024;
    L.bank_ordered = bank_classes > 0;
    const int64_t nparts = L.nparts;
    const std::vector<int64_t>& part_nnz = parts.nnz;
    L.prow0.alloc(nparts + 1);
    MX_CUDA(cudaMemcpyAsync(L.prow0.p(), parts.row0.data(), 8 * (nparts + 1), cudaMemcpyHostToDevice, st));
    DevArr<int32_t> row_part;
    row_part.alloc(std::max<int64_t>(nrows, 1));
    if (nparts > 0) {
        row_part_kernel<<<blocks_for(nparts), kThreads, 0, st>>>(L.prow0.p(), nparts, row_part.p());
        MX_LAUNCHED();
    }
    Builder b{L, nrows, ncols, R, B, R / 32, in_translate, row_part.p(), L.prow0.p(), parts.row0};
    b.bank_classes = bank_classes;
    b.col_inv = col_inv;
    b.part_class = part_class;
    b.words = std::max<int64_t>(1, ceil_div(ncols, 32));
    b.bitmap_parts = std::max<int64_t>(1, ((int64_t)2 << 30) / (b.words * 8));
    b.distinct.alloc(nparts + 1);
    b.nst.alloc(nparts + 1);
    b.slots_p.alloc(nparts + 1);
    MX_CUDA(cudaMemsetAsync(b.distinct.p(), 0, 8 * (nparts + 1), st));
    MX_CUDA(cudaMemsetAsync(b.nst.p(), 0, 8 * (nparts + 1), st));
    MX_CUDA(cudaMemsetAsync(b.slots_p.p(), 0, 8 * (nparts + 1), st));
    L.nnz = 0;
    for (int64_t v : part_nnz) L.nnz += v;
    // chunks of whole partitions under the entry budget
    std::vector<std::pair<int64_t, int64_t>> chunks;
    for (int64_t pa = 0; pa < nparts;) {
        int64_t pb = pa, acc = 0;
        while (pb < nparts && (pb == pa || acc + part_nnz[pb] <= budget)) acc += part_nnz[pb++];
        chunks.emplace_back(pa, pb);
        pa = pb;
    }
    Entries keep;
    // pass 1: sizes
    for (auto& c : chunks) {
        Entries E;
        gen(parts.row0[c.first], parts.row0[c.second], E, st);
        b.process(E, c.first, c.second, 1, st);
        if (chunks.size() == 1) keep = std::move(E);
    }
    L.stage_base.alloc(nparts + 1);
    L.map_off.alloc(nparts + 1);
    DevArr<int64_t> part_slot;
    part_slot.alloc(nparts + 1);
    exclusive_scan_i64(b.nst.p(), L.stage_base.p(), nparts + 1, st);
    exclusive_scan_i64(b.distinct.p(), L.map_off.p(), nparts + 1, st);
    exclusive_scan_i64(b.slots_p.p(), part_slot.p(), nparts + 1, st);
    b.h_stage_base = to_host(L.stage_base.p(), nparts + 1, st);
    b.h_part_slot = to_host(part_slot.p(), nparts + 1, st);
    L.nstages = b.h_stage_base[nparts];
    L.nmap = read_scalar(L.map_off.p() + nparts, st);
    L.nslots = b.h_part_slot[nparts];
    {
        const auto h_nst = to_host(b.nst.p(), nparts, st);
        int64_t mx = 1;
        for (int64_t v : h_nst) mx = std::max(mx, v);
        L.max_stages = (int32_t)mx;
    }
    const int64_t nblk = L.nstages * L.SPP;
    L.map.alloc(std::max<int64_t>(L.nmap, 1));
    L.slot_off.alloc(nblk + 1);
    MX_CUDA(cudaMemcpyAsync(L.slot_off.p() + nblk, &L.nslots, 8, cudaMemcpyHostToDevice, st));
    L.lane_chunks.alloc(std::max<int64_t>(nblk * 32, 1));
    L.ind.alloc(std::max<int64_t>(L.nslots, 1));
    L.val.alloc(std::max<int64_t>(L.nslots, 1));
    MX_CUDA(cudaMemsetAsync(L.ind.p(), 0, 2 * std::max<int64_t>(L.nslots, 1), st));
    MX_CUDA(cudaMemsetAsync(L.val.p(), 0, 4 * std::max<int64_t>(L.nslots, 1), st));
    // pass 2: scatter (regenerating each chunk unless there was only one)
    for (auto& c : chunks) {
        if (chunks.size() == 1) {
            b.process(keep, c.first, c.second, 2, st);
        } else {
            Entries E;
            gen(parts.row0[c.first], parts.row0[c.second], E, st);
            b.process(E, c.first, c.second, 2, st);
        }
    }
    if (out_translate) {
        L.out_idx.alloc(std::max<int64_t>(nrows, 1));
        MX_CUDA(cudaMemcpyAsync(L.out_idx.p(), out_translate, 4 * nrows, cudaMemcpyDeviceToDevice, st));
    }
    set_part_order(L, parts.row0, b.h_part_slot, b.h_stage_base, st);
    MX_CUDA(cudaStreamSynchronize(st));
}

// Partitions of one direction from its per-row nonzero counts.  Fixed: R rows each (reading R10,
// the paper's blocks of consecutive Hilbert rows).  Balanced (automatic tuning): still <= R
// consecutive Hilbert rows each, but cut at equal shares of the work (nonzeros + kRowCost per
// row) into a multiple of the SM count, so no SM is left with a heavier last partition -- the
// tail that left a third of the SMs idle in the single-wave A_p^T of a P = 8 rank
// (profiles/r01_virtual_scaling_cfg3.log).  Boundaries are clamped so every partition keeps
// 1..R rows.
Partitions make_partitions(const int32_t* cnt, int64_t nrows, int32_t R, bool balanced, cudaStream_t st) {
    constexpr int64_t kRowCost = 8;
    Partitions out;
    out.balanced = balanced;
    const auto h = to_host(cnt, nrows, st);
    std::vector<int64_t> w(nrows + 1, 0);
    for (int64_t r = 0; r < nrows; ++r) w[r + 1] = w[r] + h[r] + kRowCost;
    const int64_t np0 = ceil_div(nrows, (int64_t)R);
    int64_t np = np0;
    int dev = 0, sms = 148;
    MX_CUDA(cudaGetDevice(&dev));
    MX_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    // MEMXCT_BALANCE: 0 = never, 1 = only when the launch has few waves (default), 2 = always
    int mode = 1;
    if (const char* e = std::getenv("MEMXCT_BALANCE")) mode = atoi(e);
    if (mode == 1 && np0 >= 4 * (int64_t)sms) balanced = false;  // many waves: the scheduler evens out
    if (mode == 0) balanced = false;
    if (balanced && nrows > 0) {
        if (2 * np0 >= sms) np = ceil_div(np0, (int64_t)sms) * sms;
        np = std::min<int64_t>(np, nrows);
    } else {
        out.balanced = false;
    }
    out.row0.assign(np + 1, 0);
    for (int64_t j = 1; j < np; ++j) {
        int64_t b;
        if (out.balanced) {
            const double target = (double)w[nrows] * (double)j / (double)np;
            b = std::lower_bound(w.begin(), w.end(), (int64_t)std::llround(target)) - w.begin();
            b = (b + 16) / 32 * 32;  // whole warps where the clamps allow
            const int64_t prev = out.row0[j - 1];
            const int64_t lo = std::max<int64_t>(prev + 1, nrows - (np - j) * (int64_t)R);
            const int64_t hi = std::min<int64_t>(prev + R, nrows - (np - j));
            b = std::min(std::max(b, lo), hi);
        } else {
            b = std::min<int64_t>(j * (int64_t)R, nrows);
        }
        out.row0[j] = b;
    }
    out.row0[np] = nrows;
    out.nnz.assign(np, 0);
    for (int64_t p = 0; p < np; ++p)
        for (int64_t r = out.row0[p]; r < out.row0[p + 1]; ++r) out.nnz[p] += h[r];
    return out;
}

}  // namespace

// ---- slab stage order of the forward partitions (MEMXCT_OPT_STAGE_ORDER) ----------------------
// The paper cuts a partition's distinct inputs, sorted by Hilbert index, into stages (R10).  A
// stage is then a compact patch of pixels that only some of the partition's rays cross, so per
// stage only some warps (32 rays each) have work and the CTA waits at the stage barrier for the
// busiest (profiles/r01_layout_efficiency.log: 34-43 % barrier efficiency on config 5).  In slab
// order the inputs are sorted by (slab across the rays, Hilbert index): slab = floor(along /
// kSlabThick) with along = the pixel centre's coordinate along the direction (-sin phi, cos phi)
// of the partition's rays, so every stage is a band that every ray of the partition crosses.
// Directions are quantised to kSlabClasses classes phi_c = (c + 1/2) pi / C; partition p uses the
// class of its middle ray.  K_c (col -> col') and its inverse are permutations of the local
// pixels, built once per class.
constexpr int32_t kSlabClasses = 16;
constexpr double kSlabThick = 16.0;

__global__ void slab_key_kernel(const int32_t* __restrict__ tomo_nat_of_h, int64_t t0, int64_t npix, int32_t n,
                                double cphi, double sphi, uint64_t* __restrict__ key) {
    MX_LOOP(col, npix) {
        const int32_t nat = tomo_nat_of_h[t0 + col];
        const double u = (double)(nat % n) + 0.5 - 0.5 * n, v = (double)(nat / n) + 0.5 - 0.5 * n;
        const double along = -u * sphi + v * cphi;                 // |along| <= n / sqrt(2)
        const int64_t slab = (int64_t)floor(along / kSlabThick) + (int64_t)(n / kSlabThick) + 2;
        key[col] = ((uint64_t)slab << 32) | (uint64_t)col;       // (slab, Hilbert)
    }
}

__global__ void invert_kernel(const uint32_t* __restrict__ inv, int64_t n, int32_t* __restrict__ inv_out,
                              int32_t* __restrict__ fwd_out) {
    MX_LOOP(j, n) {
        inv_out[j] = (int32_t)inv[j];
        fwd_out[inv[j]] = (int32_t)j;
    }
}

// class of every forward partition: direction of its middle ray
__global__ void part_class_kernel(const int64_t* __restrict__ row0, int64_t np, const int32_t* __restrict__ hray,
                                  const int32_t* __restrict__ sino_nat_of_h, int32_t c_chan, int32_t m_proj,
                                  int32_t* __restrict__ part_class) {
    MX_LOOP(p, np) {
        const int64_t mid = (row0[p] + row0[p + 1]) / 2;
        const int32_t h = hray ? hray[mid] : (int32_t)mid;
        const int64_t m = sino_nat_of_h[h] / c_chan;
        const int64_t cl = m * kSlabClasses / m_proj;
        part_class[p] = (int32_t)(cl < kSlabClasses - 1 ? cl : kSlabClasses - 1);
    }
}

__global__ void row_class_kernel(const int64_t* __restrict__ row0, int64_t np, const int32_t* __restrict__ part_class,
                                 int32_t* __restrict__ row_class) {
    MX_LOOP(p, np)
    for (int64_t r = row0[p]; r < row0[p + 1]; ++r) row_class[r] = part_class[p];
}

// entry columns of a generated chunk -> their partition class order
__global__ void apply_class_order_kernel(const uint32_t* __restrict__ rows, int64_t n,
                                         const int32_t* __restrict__ row_class, const int32_t* __restrict__ kfwd,
                                         int64_t ncols, uint32_t* __restrict__ cols) {
    MX_LOOP(e, n) cols[e] = (uint32_t)kfwd[(int64_t)row_class[rows[e]] * ncols + cols[e]];
}

// ---- forward row grouping (MEMXCT_OPT_RAY_BLOCK) ----------------------------------------------
// Key of footprint row i: (block of `a` projections x `w` channels, then projection, channel).
// Channels are counted from shift[m] = the channel of the local tomogram's centre at projection m
// (0 for a whole tomogram centred on the rotation axis): rays of one block with equal offsets
// k - shift[m] are tangent to one circle around that centre and cross each other inside the
// local region, so the block's strips overlap there (a block with fixed channels crosses on the
// line through the rotation axis, which a rank's region need not contain).
__global__ void ray_block_key_kernel(const int32_t* __restrict__ hray, const int32_t* __restrict__ sino_nat_of_h,
                                     int64_t nrows, int32_t c, int32_t a, int32_t w,
                                     const int32_t* __restrict__ shift, uint64_t* __restrict__ key) {
    MX_LOOP(i, nrows) {
        const int32_t h = hray ? hray[i] : (int32_t)i;
        const int32_t nat = sino_nat_of_h[h];
        const int32_t m = nat / c, k = nat % c;
        const int64_t ks = (int64_t)k - shift[m] + 2 * (int64_t)c;  // >= 0
        const uint64_t blk = (uint64_t)(m / a) * (uint64_t)((4 * (int64_t)c + w - 1) / w) + (uint64_t)(ks / w);
        key[i] = (blk << 32) | (uint64_t)((int64_t)(m % a) * c + k);
    }
}

// centroid of the local pixels (integer sums: exact, so the layout is deterministic)
__global__ void centroid_kernel(const int32_t* __restrict__ tomo_nat_of_h, int64_t t0, int64_t npix, int32_t n,
                                unsigned long long* __restrict__ sums) {
    unsigned long long si = 0, sj = 0;
    MX_LOOP(q, npix) {
        const int32_t nat = tomo_nat_of_h[t0 + q];
        si += (unsigned long long)(nat / n);
        sj += (unsigned long long)(nat % n);
    }
    atomicAdd(sums, si);
    atomicAdd(sums + 1, sj);
}

// Blocked row j = footprint row perm[j]: its Hilbert ray, its length, and where its output goes
// (natural ray index, footprint position, or Hilbert index -- the plan's output order).
__global__ void ray_block_gather_kernel(const uint32_t* __restrict__ perm, const int32_t* __restrict__ hray,
                                        const int32_t* __restrict__ len, const int32_t* __restrict__ sino_nat_of_h,
                                        int64_t nrows, int mode, int32_t* __restrict__ hray_b,
                                        int32_t* __restrict__ len_b, int32_t* __restrict__ out_b) {
    MX_LOOP(j, nrows) {
        const uint32_t i = perm[j];
        const int32_t h = hray ? hray[i] : (int32_t)i;
        hray_b[j] = h;
        len_b[j] = len[i];
        out_b[j] = mode == 0 ? sino_nat_of_h[h] : mode == 1 ? (int32_t)i : h;
    }
}

// MEMXCT_OPT_RAY_BLOCK resolved: projections per forward row block, or -1 (Hilbert rows).
// A partition of R rays that spans `a` projections and R/a channels touches about the fewest
// distinct pixels when the angular fan of the block across the local tomogram (side L, angle step
// pi/M, so (a-1) L pi/M pixels of drift) is comparable to its width R/a: a* = sqrt(R / (L pi / M)).
// The paper's Hilbert rows form ~sqrt(R) x sqrt(R) squares, which is that optimum when L pi/M ~ 1
// (configs 1-4: 2.1-2.7); blocks are used only when a* is >= 4x smaller (config 5: L pi/M ~ 35-99).
// Measured (profiles/r01_ray_block_sweep.md): whole tomograms 2048^2 / 60 and 4096^2 / 180
// (a* = 3.1, 3.8) are fastest at a = 8, config-5 shards (a* = 5.35, blocks sheared onto the
// rank's region, ray_block_key_kernel) at a = 16 (8.0 ms vs 8.6 at a = 8 and 8.8 at a = 32):
// the smallest power of two >= 2 a* in all three.  (The earlier factor 3 for decomposed plans
// gave a = 32 at a* = 5.35: profiles/r01h_shard_cfg5_p8.jsonl.)
int32_t resolve_ray_block(const Plan& P, int64_t local_pixels, int32_t R) {
    if (P.opt.canonical || P.opt.ray_block < 0) return -1;
    int32_t a = (int32_t)P.opt.ray_block;
    if (a == 0) {
        const double drift = std::sqrt((double)std::max<int64_t>(local_pixels, 1)) * M_PI / (double)P.m;
        const double astar = std::sqrt((double)R / std::max(drift, 1e-9));
        if (astar > std::sqrt((double)R) / 4.0) return -1;
        a = 1;
        while (a < 2.0 * astar && a * 2 <= R / 32) a *= 2;
    }
    return std::min<int32_t>(a, std::max(1, R / 32));
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

    PhaseClock clk(P.build_s, st);
    // a3: this rank's tomogram and sinogram subdomains (whole domains at P = 1)
    decompose(P, G, st);
    const int64_t npix = P.t1 - P.t0;
    clk.mark(kPhDecompose);

    // rows of A_p = footprint rays (every ray at P = 1) and their lengths
    DevArr<int32_t> fp_len;
    const int64_t nrows = P.nfp = footprint(P, G, fp_len, st);
    clk.mark(kPhCount);
    const int32_t* hray = !P.dist ? nullptr : P.fp_rays.p();
    const bool natural = (P.opt.vector_order == 0);  // P = 1 only
    int32_t R, B, Rb, Bb;
    resolve_tuning(P, nrows, &R, &B);  // A_p: rows = footprint rays
    resolve_tuning(P, npix, &Rb, &Bb);  // A_p^T: rows = local pixels
    P.part_rows = R;
    P.buffer_entries = B;
    if (P.opt.precision == 1) {  // fp64 stage buffer: half the entries
        B /= 2;
        Bb /= 2;
    }

    // forward rows grouped into projection x channel blocks (MEMXCT_OPT_RAY_BLOCK), or the
    // footprint's Hilbert order; the A_p^T build below keeps the footprint order for its columns
    P.ray_block = resolve_ray_block(P, npix, R);
    // drifting stages (spmv_f32_drift_kernel) for the forward operator of projection-block plans:
    // three stage buffers of 13312 entries (16384 until r02aw) instead of one of 36 R.  Config-5 shard forward 7.99 ->
    // 7.73 ms although the smaller stages add 2.2 % slab padding; the balanced back operator and
    // the Hilbert-row geometries (configs 1-4) gain nothing and keep the plain kernel
    // (profiles/r01i_drift_*.jsonl).  MEMXCT_DRIFT=1 forces it for both directions.
    const bool fwd_drift = drift_requested() || (P.ray_block > 0 && P.opt.buffer_entries == 0 &&
                                                 P.opt.precision == 0 && P.opt.slices <= 1);
    if (fwd_drift && P.opt.buffer_entries == 0) {
        B = std::min(B, drift_auto_b());
        P.buffer_entries = B;
    }
    DevArr<int32_t> hray_b, len_b, out_b;
    const int32_t* fwd_hray = hray;
    const int32_t* fwd_len = fp_len.p();
    const int32_t* fwd_out = natural ? P.sino_nat_of_h.p() : nullptr;
    if (P.ray_block > 0 && nrows > 1) {
        const int32_t a = P.ray_block, w = std::max(1, R / a);
        DevArr<uint64_t> key, key_s;
        DevArr<uint32_t> idx, perm;
        key.alloc(nrows);
        key_s.alloc(nrows);
        idx.alloc(nrows);
        perm.alloc(nrows);
        // channel of the local tomogram's centre per projection (all 0 for the whole tomogram)
        std::vector<int32_t> h_shift(P.m, 0);
        if (P.dist && npix > 0) {
            DevArr<unsigned long long> sums;
            sums.alloc(2);
            MX_CUDA(cudaMemsetAsync(sums.p(), 0, 16, st));
            centroid_kernel<<<blocks_for(npix), kThreads, 0, st>>>(P.tomo_nat_of_h.p(), P.t0, npix, P.n, sums.p());
            MX_LAUNCHED();
            const auto hs = to_host(sums.p(), 2, st);
            const double cy = (double)hs[0] / npix + 0.5 - 0.5 * P.n, cx = (double)hs[1] / npix + 0.5 - 0.5 * P.n;
            for (int32_t mm = 0; mm < P.m; ++mm) {
                const double th = (double)mm * M_PI / (double)P.m;
                h_shift[mm] = (int32_t)std::lround(cx * std::cos(th) + cy * std::sin(th));
            }
        }
        DevArr<int32_t> shift;
        shift.alloc(P.m);
        MX_CUDA(cudaMemcpyAsync(shift.p(), h_shift.data(), 4 * P.m, cudaMemcpyHostToDevice, st));
        ray_block_key_kernel<<<blocks_for(nrows), kThreads, 0, st>>>(hray, P.sino_nat_of_h.p(), nrows, P.c, a, w,
                                                                     shift.p(), key.p());
        MX_LAUNCHED();
        iota_kernel<uint32_t><<<blocks_for(nrows), kThreads, 0, st>>>(idx.p(), nrows);
        MX_LAUNCHED();
        size_t tb = 0;
        MX_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, key.p(), key_s.p(), idx.p(), perm.p(), (int)nrows, 0, 64, st));
        DevBuf tmp(tb);
        MX_CUDA(cub::DeviceRadixSort::SortPairs(tmp.get(), tb, key.p(), key_s.p(), idx.p(), perm.p(), (int)nrows, 0, 64, st));
        MX_LAUNCHED();
        hray_b.alloc(nrows);
        len_b.alloc(nrows);
        out_b.alloc(nrows);
        const int mode = natural ? 0 : (P.dist ? 1 : 2);
        ray_block_gather_kernel<<<blocks_for(nrows), kThreads, 0, st>>>(perm.p(), hray, fp_len.p(), P.sino_nat_of_h.p(),
                                                                        nrows, mode, hray_b.p(), len_b.p(), out_b.p());
        MX_LAUNCHED();
        fwd_hray = hray_b.p();
        fwd_len = len_b.p();
        fwd_out = out_b.p();
    }

    // equal-work partitions only under the automatic tuning (PART_ROWS given: the user's fixed
    // blocks; CANONICAL: the oracle's fixed R-row dot chunks)
    const bool balance = P.opt.part_rows == 0 && !P.opt.canonical;
    const Partitions fwd_parts = make_partitions(fwd_len, nrows, R, balance, st);

    // slab stage order (MEMXCT_OPT_STAGE_ORDER): per-class column orders, class of every partition
    // and row; auto = slab order in FP32 mode (cfg3 forward 1.733 -> 1.714 ms, cfg4 10.86 ->
    // 10.74 ms, config-5 shards 2-3x, profiles/r01_slab_stages.md); MIXED keeps the Hilbert
    // stages, whose fp64 row chains ascend in Hilbert input order like the oracle's (R16)
    P.stage_order = (P.opt.canonical || P.opt.stage_order < 0) ? -1
                    : (P.opt.stage_order > 0 || P.opt.precision == 0) ? 1 : -1;
    DevArr<int32_t> kfwd, kinv, part_class, row_class;
    const int64_t fnp = (int64_t)fwd_parts.row0.size() - 1;
    if (P.stage_order == 1 && npix > 0 && nrows > 0) {
        kfwd.alloc((int64_t)kSlabClasses * npix);
        kinv.alloc((int64_t)kSlabClasses * npix);
        DevArr<uint64_t> key, key_s;
        DevArr<uint32_t> idx, inv;
        key.alloc(npix);
        key_s.alloc(npix);
        idx.alloc(npix);
        inv.alloc(npix);
        size_t tb = 0;
        MX_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tb, key.p(), key_s.p(), idx.p(), inv.p(), (int)npix, 0, 64, st));
        DevBuf tmp(tb);
        for (int32_t cl = 0; cl < kSlabClasses; ++cl) {
            const double phi = (cl + 0.5) * M_PI / kSlabClasses;
            slab_key_kernel<<<blocks_for(npix), kThreads, 0, st>>>(P.tomo_nat_of_h.p(), P.t0, npix, P.n, std::cos(phi),
                                                                   std::sin(phi), key.p());
            MX_LAUNCHED();
            iota_kernel<uint32_t><<<blocks_for(npix), kThreads, 0, st>>>(idx.p(), npix);
            MX_LAUNCHED();
            MX_CUDA(cub::DeviceRadixSort::SortPairs(tmp.get(), tb, key.p(), key_s.p(), idx.p(), inv.p(), (int)npix, 0, 64, st));
            MX_LAUNCHED();
            invert_kernel<<<blocks_for(npix), kThreads, 0, st>>>(inv.p(), npix, kinv.p() + cl * npix, kfwd.p() + cl * npix);
            MX_LAUNCHED();
        }
        DevArr<int64_t> row0;
        row0.alloc(fnp + 1);
        MX_CUDA(cudaMemcpyAsync(row0.p(), fwd_parts.row0.data(), 8 * (fnp + 1), cudaMemcpyHostToDevice, st));
        part_class.alloc(std::max<int64_t>(fnp, 1));
        row_class.alloc(nrows);
        part_class_kernel<<<blocks_for(fnp), kThreads, 0, st>>>(row0.p(), fnp, fwd_hray, P.sino_nat_of_h.p(), P.c, P.m,
                                                                part_class.p());
        MX_LAUNCHED();
        row_class_kernel<<<blocks_for(fnp), kThreads, 0, st>>>(row0.p(), fnp, part_class.p(), row_class.p());
        MX_LAUNCHED();
        MX_CUDA(cudaStreamSynchronize(st));
    }
    int64_t nnz = 0;
    for (int64_t v : fwd_parts.nnz) nnz += v;
    const int64_t budget = chunk_budget(2 * nnz);
    // bank-aware run order for FP32 plans tuned for batched calls (16 B entries: 8 lanes per
    // shared-memory phase; 8 B: 16); canonical order (ascending) otherwise
    const int32_t bank = (P.opt.precision == 0 && P.opt.slices > 1) ? (P.opt.slices > 2 ? 8 : 16) : 0;

    // ---- A_p: rows = footprint rays; entries of each ray sorted by local pixel --------------
    double gen_s = 0.0;  // generator time inside build_direction (charged to trace / sort)
    Generator gen_fwd = [&](int64_t ra, int64_t rb, Entries& E, cudaStream_t s) {
        EventSplit ev;
        const int64_t nr = rb - ra;
        DevArr<int64_t> len64, rp;
        len64.alloc(nr + 1);
        rp.alloc(nr + 1);
        widen_i32_to_i64(fwd_len + ra, len64.p(), nr, s);
        MX_CUDA(cudaMemsetAsync(len64.p() + nr, 0, 8, s));
        exclusive_scan_i64(len64.p(), rp.p(), nr + 1, s);
        E.n = read_scalar(rp.p() + nr, s);
        DevArr<uint32_t> col;
        DevArr<float> val;
        col.alloc(std::max<int64_t>(E.n, 1));
        val.alloc(std::max<int64_t>(E.n, 1));
        E.row.alloc(std::max<int64_t>(E.n, 1));
        ev.rec(0, s);
        trace_emit(P, G, fwd_hray, ra, nr, P.t0, P.t1, rp.p(), col.p(), val.p(), E.row.p(), s);
        ev.rec(1, s);
        if (kfwd.p() && E.n > 0) {  // slab stage order: sort each row by its partition's class order
            apply_class_order_kernel<<<blocks_for(E.n), kThreads, 0, s>>>(E.row.p(), E.n, row_class.p(), kfwd.p(),
                                                                          npix, col.p());
            MX_LAUNCHED();
        }
        E.col.alloc(std::max<int64_t>(E.n, 1));
        E.val.alloc(std::max<int64_t>(E.n, 1));
        if (E.n > 0) {
            size_t tb = 0;
            MX_CUDA(cub::DeviceSegmentedSort::SortPairs(nullptr, tb, col.p(), E.col.p(), val.p(), E.val.p(),
                                                        (int)E.n, (int)nr, rp.p(), rp.p() + 1, s));
            DevBuf tmp(tb);
            MX_CUDA(cub::DeviceSegmentedSort::SortPairs(tmp.get(), tb, col.p(), E.col.p(), val.p(), E.val.p(),
                                                        (int)E.n, (int)nr, rp.p(), rp.p() + 1, s));
            MX_LAUNCHED();
        }
        ev.rec(2, s);
        MX_CUDA(cudaStreamSynchronize(s));
        const double before = P.build_s[kPhTraceFwd] + P.build_s[kPhSortFwd];
        ev.charge(P.build_s, kPhTraceFwd, kPhSortFwd);
        gen_s += P.build_s[kPhTraceFwd] + P.build_s[kPhSortFwd] - before;
    };
    build_direction(P.fwd, nrows, npix, fwd_parts, R, B, gen_fwd, natural ? P.tomo_nat_of_h.p() : nullptr,
                    fwd_out, budget, bank, st, kinv.p(), part_class.p());
    clk.mark(kPhLayoutFwd);
    P.build_s[kPhLayoutFwd] -= gen_s;  // the generator's share is in trace / sort
    P.fwd.drift = fwd_drift && 12 * (int64_t)B <= 224 * 1024;
    if (rle_requested()) encode_map_runs(P.fwd, st);
    kfwd.reset();
    kinv.reset();
    part_class.reset();
    row_class.reset();
    hray_b.reset();
    len_b.reset();
    out_b.reset();

    // ---- A_p^T: rows = local pixels; every footprint ray re-traced with the chunk's pixel range,
    // then the order-preserving (stable) sort by pixel -------------------------------------------
    DevArr<int32_t> pix_cnt;
    pix_cnt.alloc(std::max<int64_t>(npix, 1));
    MX_CUDA(cudaMemsetAsync(pix_cnt.p(), 0, 4 * std::max<int64_t>(npix, 1), st));
    trace_hist(P, G, hray, 0, nrows, P.t0, P.t1, true, pix_cnt.p(), st);
    clk.mark(kPhTraceBack);
    const Partitions back_parts = make_partitions(pix_cnt.p(), npix, Rb, balance, st);
    pix_cnt.reset();
    gen_s = 0.0;
    Generator gen_back = [&](int64_t ra, int64_t rb, Entries& E, cudaStream_t s) {
        EventSplit ev;
        ev.rec(0, s);
        const int64_t lo = P.t0 + ra, hi = P.t0 + rb;
        DevArr<int32_t> len;
        len.alloc(std::max<int64_t>(nrows, 1));
        trace_count(P, G, hray, 0, nrows, lo, hi, true, len.p(), s);
        DevArr<int64_t> len64, rp;
        len64.alloc(nrows + 1);
        rp.alloc(nrows + 1);
        widen_i32_to_i64(len.p(), len64.p(), nrows, s);
        MX_CUDA(cudaMemsetAsync(len64.p() + nrows, 0, 8, s));
        exclusive_scan_i64(len64.p(), rp.p(), nrows + 1, s);
        len.reset();
        len64.reset();
        E.n = read_scalar(rp.p() + nrows, s);
        DevArr<uint32_t> pix, ray;
        DevArr<float> val;
        pix.alloc(std::max<int64_t>(E.n, 1));
        ray.alloc(std::max<int64_t>(E.n, 1));
        val.alloc(std::max<int64_t>(E.n, 1));
        trace_emit(P, G, hray, 0, nrows, lo, hi, rp.p(), pix.p(), val.p(), ray.p(), s);
        ev.rec(1, s);
        rp.reset();
        DevArr<uint32_t> perm;
        E.row.alloc(std::max<int64_t>(E.n, 1));
        perm.alloc(std::max<int64_t>(E.n, 1));
        if (E.n > 0) stable_sort_by_key(pix.p(), E.row.p(), perm.p(), E.n, std::max<int64_t>(rb - ra, 1), s);
        pix.reset();
        E.col.alloc(std::max<int64_t>(E.n, 1));
        E.val.alloc(std::max<int64_t>(E.n, 1));
        if (E.n > 0) {
            gather_u32_f32<<<blocks_for(E.n), kThreads, 0, s>>>(perm.p(), ray.p(), val.p(), E.col.p(), E.val.p(), E.n);
            MX_LAUNCHED();
            offset_u32_kernel<<<blocks_for(E.n), kThreads, 0, s>>>(E.row.p(), E.n, (uint32_t)ra);
            MX_LAUNCHED();
        }
        ev.rec(2, s);
        MX_CUDA(cudaStreamSynchronize(s));
        const double before = P.build_s[kPhTraceBack] + P.build_s[kPhTranspose];
        ev.charge(P.build_s, kPhTraceBack, kPhTranspose);
        gen_s += P.build_s[kPhTraceBack] + P.build_s[kPhTranspose] - before;
    };
    build_direction(P.back, npix, nrows, back_parts, Rb, Bb, gen_back, natural ? P.sino_nat_of_h.p() : nullptr,
                    natural ? P.tomo_nat_of_h.p() : nullptr, chunk_budget(nnz), bank, st);
    if (rle_requested()) encode_map_runs(P.back, st);
    clk.mark(kPhLayoutBack);
    P.build_s[kPhLayoutBack] -= gen_s;

    // a6: exchange maps of the sparse all-to-allv (P > 1)
    if (P.shard) shard_receive_maps(P, G, st);
    build_exchange(P, st);
    clk.mark(kPhExchange);
}

}  // namespace mx
