// plan.h -- internal plan and layout structures of libmemxct.
#pragma once

#include <map>
#include <memory>
#include <tuple>
#include <vector>

#include "common.h"

namespace mx {

// One SpMV direction (A: rows = rays, cols = pixels; A^T: rows = pixels, cols = rays) in the
// staged SELL-32 layout (Listing 3; padding per 32-row warp slice, reading R11).
//
//   partition p (one CTA)      rows [p*R, p*R + R) in plan (Hilbert) order
//   its stages                 global indices [stage_base[p], stage_base[p+1])
//   stage-buffer map           map[map_off[p] + s*B + i] = input index of buffer slot i of
//                              local stage s (distinct inputs of p sorted by Hilbert index, cut
//                              into chunks of B, reading R10)
//   (stage g, slice w) block   slots [slot_off[g*SPP + w], slot_off[g*SPP + w + 1]).
//                              Lane l (row w*32 + l) owns n_l = lane_chunks[(g*SPP + w)*32 + l]
//                              chunks of kVec slots (its run length rounded up to kVec).
//                              "Jagged SELL": chunk c is stored only for the a_c lanes with
//                              n_l > c, packed in lane order; chunk c starts after
//                              prefix_c = sum_l min(n_l, c) chunks.  Inside chunk c:
//                                ind: [a_c lanes][kVec] uint16        (16 B per lane)
//                                val: [kVec/4][a_c lanes][4] fp32     (2 x 16 B per lane)
//                              so the active lanes of a warp read contiguous, fully coalesced
//                              16 B vectors and no padding beyond the per-lane round-up to kVec
//                              is stored or streamed (padding slots: ind 0, val 0).
//   entries of a row in a stage ascend by local index (= ascending Hilbert input index).
struct Layout {
    int64_t nrows = 0, ncols = 0, nnz = 0;
    int64_t nparts = 0, nstages = 0, nslots = 0, nmap = 0;
    int32_t R = 0, SPP = 0, B = 0;
    int32_t max_stages = 0;
    DevArr<int64_t> stage_base;  // nparts + 1
    DevArr<int64_t> map_off;     // nparts + 1
    DevArr<int32_t> map;         // nmap
    DevArr<int64_t> slot_off;    // nstages * SPP + 1
    DevArr<uint16_t> ind;        // nslots
    DevArr<float> val;           // nslots
    DevArr<uint16_t> lane_chunks;  // nstages * SPP * 32
    DevArr<int32_t> out_idx;     // nrows, optional: output position of each row (natural order)
    int64_t device_bytes() const {
        return (int64_t)(stage_base.buf.bytes() + map_off.buf.bytes() + map.buf.bytes() +
                         slot_off.buf.bytes() + ind.buf.bytes() + val.buf.bytes() +
                         lane_chunks.buf.bytes() + out_idx.buf.bytes());
    }
};

constexpr int kVec = 8;  // SELL column chunk: 8 slots per lane per chunk

struct Options {
    int64_t tile_tomo = 0;  // 0 = default rule R7
    int64_t tile_sino = 0;
    int64_t part_rows = 0;       // 0 = auto (resolve_tuning)
    int64_t buffer_entries = 0;  // 0 = auto (resolve_tuning)
    int64_t precision = 0;  // 0 FP32, 1 MIXED
    int64_t canonical = 0;
    int64_t cg_variant = 0;
    int64_t vector_order = 0;  // 0 natural, 1 plan
};

struct CgGraph {
    cudaGraphExec_t exec = nullptr;
    int64_t nkernels = 0;
    ~CgGraph() { if (exec) cudaGraphExecDestroy(exec); }
};

struct Plan {
    int32_t n = 0, m = 0, c = 0;
    Options opt;
    bool built = false;
    int32_t rank = 0, nranks = 1, device = -1;
    int32_t tile_tomo = 0, tile_sino = 0;
    bool fused_dot = false;  // MEMXCT_FUSED_DOT=1: fuse CG dots into the SpMV epilogue (tuning)
    int32_t part_rows = 0, buffer_entries = 0;  // resolved tuning (build)

    // two-level pseudo-Hilbert permutations, device int32
    DevArr<int32_t> tomo_nat_of_h, tomo_h_of_nat;  // N*N
    DevArr<int32_t> sino_nat_of_h, sino_h_of_nat;  // M*C

    Layout fwd;   // A   (forward projection)
    Layout back;  // A^T (backprojection)

    // CG state (element size 4 in FP32 mode, 8 in MIXED mode)
    size_t esize = 4;
    DevBuf cg_r, cg_q, cg_s, cg_p, cg_ax;      // vectors
    DevArr<double> part_fwd, part_back, part_vec;  // per-CTA dot partials
    DevArr<double> scal;                            // per-iteration scalars
    DevArr<unsigned int> tickets;                   // last-block counters
    int64_t scal_iters = -1;
    // staging for *_host calls
    DevBuf h_in, h_out;
    std::map<std::tuple<const void*, void*, int32_t, cudaStream_t>, std::unique_ptr<CgGraph>> graphs;

    int64_t vec_len(int domain) const { return domain == 0 ? (int64_t)n * n : (int64_t)m * c; }
    int64_t device_bytes() const;
};

// hilbert.cu
void build_hilbert(int32_t h, int32_t w, int32_t t, int32_t* nat_of_h, int32_t* h_of_nat,
                   cudaStream_t st);
int32_t default_tile(int32_t h, int32_t w);

// trace.cu: Siddon count / emit over rays listed in plan (Hilbert) order
void trace_count(const Plan& P, const double* cos_t, const double* sin_t, int64_t nrays,
                 int32_t* row_len, cudaStream_t st);
void trace_emit(const Plan& P, const double* cos_t, const double* sin_t, int64_t nrays,
                const int64_t* row_ptr, uint32_t* cols, float* vals, uint32_t* row_ids,
                cudaStream_t st);

// layout.cu: staged SELL-32 layout from entries sorted by (row, col)
void build_layout(Layout& L, int64_t nrows, int64_t ncols, int64_t nnz, const uint32_t* row_ids,
                  const uint32_t* cols, const float* vals, int32_t R, int32_t B,
                  const int32_t* in_translate, const int32_t* out_translate, cudaStream_t st);
void build_matrices(Plan& P, cudaStream_t st);

// spmv.cu
void spmv_init();
void spmv_f32(const Layout& L, const float* x, float* y, double* dot_part, double* dot_out,
              unsigned int* ticket, cudaStream_t st);
void spmv_f64(const Layout& L, const double* x, double* y, double* dot_part, double* dot_out,
              unsigned int* ticket, bool canonical, cudaStream_t st);

// cg.cu
void cg_run(Plan& P, const void* y, void* x, int32_t iters, cudaStream_t st);
void cg_fetch_norms(Plan& P, int32_t iters, double* out, cudaStream_t st);

}  // namespace mx
