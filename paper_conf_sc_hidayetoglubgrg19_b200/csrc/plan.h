// plan.h -- internal plan and layout structures of libmemxct.
#pragma once

#include <chrono>
#include <map>
#include <memory>
#include <tuple>
#include <vector>

#include "comm.h"
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
    bool bank_ordered = false;   // runs in bank-aware order instead of ascending local index
    bool balanced = false;       // partitions cut for equal work (else fixed R rows each)
    bool drift = false;          // FP32 single-slice launches use spmv_f32_drift_kernel
    DevArr<int64_t> prow0;       // nparts + 1: first row of each partition (<= R rows each)
    DevArr<int64_t> stage_base;  // nparts + 1
    DevArr<int64_t> map_off;     // nparts + 1
    DevArr<int32_t> map;         // nmap
    DevArr<int64_t> slot_off;    // nstages * SPP + 1
    DevArr<uint16_t> ind;        // nslots
    DevArr<float> val;           // nslots
    DevArr<uint16_t> lane_chunks;  // nstages * SPP * 32
    DevArr<int32_t> out_idx;     // nrows, optional: output position of each row (natural order)
    DevArr<int32_t> part_order;  // nparts, optional: partition run by CTA b (launch order)
    int64_t n_first = -1;        // P > 1 forward: the first n_first CTAs hold every partition with
                                 // rows owned by other ranks (exchange overlap), else -1
    // Run-length stage maps (rle.cu, MEMXCT_RLE): every 32-slot block of a stage's map as one
    // 16 B record of up to 4 runs of consecutive input indices -- start | (first slot << 27) per
    // run -- instead of 32 int32 entries; blocks with more runs hold (1 << 27) | overflow block
    // and keep their 32 entries in `ovf`.  The stage gather reads a record (broadcast) per 32
    // slots: 0.5 B per map entry plus overflow instead of 4 B.
    bool rle = false;
    DevArr<int64_t> blk_base;    // nstages + 1: first 32-slot block of every stage
    DevArr<int4> blk_rec;        // one record per block
    DevArr<int32_t> ovf;         // 32 entries per overflow block
    int64_t n_ovf = 0;
    int64_t device_bytes() const {
        return (int64_t)(prow0.buf.bytes() + stage_base.buf.bytes() + map_off.buf.bytes() + map.buf.bytes() +
                         slot_off.buf.bytes() + ind.buf.bytes() + val.buf.bytes() +
                         lane_chunks.buf.bytes() + out_idx.buf.bytes() + part_order.buf.bytes() +
                         blk_base.buf.bytes() + blk_rec.buf.bytes() + ovf.buf.bytes());
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
    int64_t slices = 1;        // slices per batched call the stage buffer is sized for
    int64_t exchange = 0;      // P > 1: 0 = transport collectives (NCCL), 1 = fused peer memory
    int64_t ray_block = 0;     // forward partitions: -1 Hilbert rows, a > 0 blocks of a projections, 0 auto
    int64_t stage_order = 0;   // forward stages: -1 Hilbert (paper), 1 slabs across the rays, 0 auto
};

// host-side angle tables on the device (reading R1)
struct Geometry {
    const double* cos_t = nullptr;
    const double* sin_t = nullptr;
};

// Arguments of the fused SpMV + exchange epilogue and of the peer-memory pack (P > 1)
constexpr int kMaxPeers = 16;
constexpr int kMaxDotSlices = 64;  // slices per CG call (cg_run's K bound)
struct PeerArgs {
    int32_t P = 0, me = 0;
    int64_t bound[kMaxPeers + 1] = {};           // row ranges per destination rank
    float* dst[kMaxPeers] = {};                  // destination buffer of rank h (peer pointer)
    int64_t off[kMaxPeers] = {};                 // element offset: dst[h][off[h] + row]
    unsigned long long* flag[kMaxPeers] = {};    // flag array of rank h (peer pointer)
    unsigned long long* my_flags = nullptr;      // this rank's flag array
    unsigned int* ticket = nullptr;              // last-CTA counter
    int32_t slot = 0;                            // arrival slot base in the peers' flag arrays
    int32_t epoch_index = 0;                     // this rank's epoch counter in my_flags
    // Folded synchronisation (NCCL ranks, one GPU each): the kernel itself waits for my_flags
    // [wait_base, wait_base + P) to reach the epoch (thread 0 of every CTA, before the data it
    // guards is touched) and, for the back SpMV, publishes the credits from its last CTA --
    // instead of separate one-thread wait / signal kernels.  Off for virtual ranks: P ranks'
    // kernels share one GPU there, and CTAs spinning on every SM could keep a peer's kernel from
    // ever being scheduled.
    int32_t fold = 0;
    int32_t wait_base = 0;
    unsigned int* abort = nullptr;               // peer_abort_word(): set by a timed-out wait
    // CG dot summed over the ranks by the kernel's last CTA (folded peer dot, one slice): the
    // peer_allreduce protocol of peer.cu on one value, in place of its one-thread kernel
    int32_t dot_fold = 0;
    double* dot_dst[kMaxPeers] = {};               // rank q's dot slots (peer pointer)
    unsigned long long* dot_flag[kMaxPeers] = {};  // rank q's dot flags (peer pointer)
    const double* dot_mine = nullptr;              // my dot slots
    unsigned long long* dot_my_flags = nullptr;    // my dot flags: [P arrivals | epoch]
};

// A process-wide word in mapped (device-visible) host memory: a peer-flag wait that times out
// (a peer is gone) sets it and returns instead of trapping, every other wait then gives up at
// once, and the host reports MEMXCT_ERR_NCCL at the next call on a decomposed plan
// (check_peer_abort).  The results of the interrupted call are undefined.
unsigned int* peer_abort_word();
void check_peer_abort();

#ifdef __CUDACC__
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// One thread: wait until flags[base + q] >= target for q < P.  After ~20 s (a peer is gone), or
// as soon as another wait has given up, set / see *abort and return instead of hanging (the
// host turns it into MEMXCT_ERR_NCCL; check_peer_abort).
__device__ inline void wait_flags(const unsigned long long* flags, int base, int P, unsigned long long target,
                                  int me, unsigned int* abort) {
    const long long t0 = clock64();
    unsigned polls = 0;
    for (int q = 0; q < P; ++q) {
        while (ld_acquire_sys(flags + base + q) < target) {
            __nanosleep(64);
            if ((++polls & 4095u) == 0 && abort && *(volatile unsigned int*)abort) return;
            if (clock64() - t0 > 40000000000LL) {
                printf("memxct peer wait timeout: rank %d base %d q %d target %llu value %llu\n", me, base, q,
                       target, ld_acquire_sys(flags + base + q));
                if (abort) {
                    *(volatile unsigned int*)abort = 1u;
                    __threadfence_system();
                }
                return;
            }
        }
    }
}
#endif

#ifdef __CUDACC__
// One thread (a kernel's last CTA): *v summed over the ranks in rank order through peer memory
// (the protocol of peer.cu: peer_allreduce_kernel, kMaxDotSlices slots per parity).
__device__ inline void peer_dot_allreduce(const PeerArgs& pa, double* v) {
    const unsigned long long e = pa.dot_my_flags[pa.P] + 1;
    pa.dot_my_flags[pa.P] = e;
    const int par = (int)(e & 1ull);
    const double mine = *v;
    for (int q = 0; q < pa.P; ++q) pa.dot_dst[q][((int64_t)par * pa.P + pa.me) * kMaxDotSlices] = mine;
    __threadfence_system();
    for (int q = 0; q < pa.P; ++q) st_release_sys(pa.dot_flag[q] + pa.me, e);
    wait_flags(pa.dot_my_flags, 0, pa.P, e, pa.me, pa.abort);
    const volatile double* m = pa.dot_mine + (int64_t)par * pa.P * kMaxDotSlices;
    double acc = m[0];
    for (int q = 1; q < pa.P; ++q) acc += m[(int64_t)q * kMaxDotSlices];
    *v = acc;
}
#endif

// sparse all-to-allv plan of this rank (P > 1)
struct Exchange {
    // forward: partials of footprint slice [sdispl[h], sdispl[h+1]) go to ray owner h;
    // partials from peer q land in recv_buf[rdispl[q] .. + rcount[q]).  Back reverses both.
    std::vector<int64_t> scount, sdispl, rcount, rdispl;
    int64_t nrecv = 0;
    DevArr<int32_t> recv_idx;  // owned-local ray of every received partial (peer order)
    DevArr<int64_t> red_ptr;   // reduction map R: CSR over owned rays ...
    DevArr<int32_t> red_pos;   // ... of positions in recv_buf, ascending peer order
    DevBuf y_fp, recv_buf;     // footprint partials, receive / pack buffer
    DevBuf y_fp_b, recv_b;     // the same for batched (multi-slice) calls
    int32_t batch_cap = 0;
    // dense collectives (EXCHANGE = 2): footprint partials scattered into a zeroed [P][maxown]
    // sinogram (rank h's owned rays, Hilbert order, padded to the largest range), reduce-scatter;
    // back: allgather of the owned values into it, gather of the footprint
    bool dense = false;
    int64_t maxown = 0;
    DevArr<int32_t> dense_pos;  // nfp: position of footprint row i in the dense sinogram
    DevBuf dense_buf, dense_own;
    // fused peer-memory exchange (EXCHANGE = 1): peers' buffers and flags mapped into this rank
    bool peer = false;
    DevArr<unsigned long long> flags;  // [4P + 2]: arrivals fwd | arrivals back | credits fwd |
                                       // credits back | my fwd epoch | my back epoch
    std::vector<void*> peer_recv, peer_yfp, peer_flags;
    std::vector<int64_t> fwd_off;      // owner h: my partial of footprint row i goes to recv_h[fwd_off[h] + i]
    std::vector<int64_t> back_off;     // peer g: my value j (recv order) goes to yfp_g[back_off[g] + j]
    // CG dots over peer memory (peer_allreduce): values [2 parities][P][kMaxDotSlices] and flags
    // [P arrivals | my epoch], mapped into every rank
    DevArr<double> dotx;
    DevArr<unsigned long long> dflags;
    std::vector<void*> peer_dotx, peer_dflags;
    DevArr<double> dot_part;           // per-CTA partials of the fused reduce + dot / A_p^T dot
    DevArr<unsigned int> tickets;      // last-CTA counters: 0 A_p remote, 1 pack, 2 reduce, 3 A_p^T
                                       // credits, 4 A_p^T dot
    bool fold = false;                 // folded waits / signals (NCCL ranks; PeerArgs::fold)
    // forward overlap (sparse collective exchange): side stream for the self-owned partitions
    cudaStream_t side = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    Exchange() = default;
    Exchange(const Exchange&) = delete;
    Exchange& operator=(const Exchange&) = delete;
    ~Exchange() {
        if (ev_fork) cudaEventDestroy(ev_fork);
        if (ev_join) cudaEventDestroy(ev_join);
        if (side) cudaStreamDestroy(side);
    }
    int64_t device_bytes() const {
        return (int64_t)(recv_idx.buf.bytes() + red_ptr.buf.bytes() + red_pos.buf.bytes() + y_fp.bytes() +
                         recv_buf.bytes() + y_fp_b.bytes() + recv_b.bytes() + dense_pos.buf.bytes() +
                         dense_buf.bytes() + dense_own.bytes());
    }
};

// SIRT scratch (sirt.cu): inverse row / column sums and work vectors
struct SirtState {
    bool ready = false;
    DevBuf rinv, cinv, r, ax, s, ones;
    DevArr<double> part;
    int64_t device_bytes() const {
        return (int64_t)(rinv.bytes() + cinv.bytes() + r.bytes() + ax.bytes() + s.bytes() + ones.bytes() +
                         part.buf.bytes());
    }
};

constexpr size_t kMaxGraphs = 8;
struct CgGraph {
    cudaGraphExec_t exec = nullptr;
    int64_t nkernels = 0;
    int64_t last_used = 0;
    ~CgGraph() { if (exec) cudaGraphExecDestroy(exec); }
};

// Wall-clock seconds of the build phases (memxct_build_phases; NEXT-3).  Phases are
// separated by stream synchronisations the build has anyway, and inside the chunk generators by
// CUDA events, so timing adds no synchronisation.
enum BuildPhase {
    kPhHilbert = 0, kPhDecompose, kPhCount, kPhTraceFwd, kPhSortFwd, kPhLayoutFwd, kPhTraceBack,
    kPhTranspose, kPhLayoutBack, kPhExchange, kPhTotal, kNumPhases
};
struct PhaseClock {
    double* acc;
    cudaStream_t st;
    std::chrono::steady_clock::time_point t;
    PhaseClock(double* a, cudaStream_t s) : acc(a), st(s), t(std::chrono::steady_clock::now()) {}
    // synchronise, charge the time since the last mark to `phase`
    void mark(int phase) {
        MX_CUDA(cudaStreamSynchronize(st));
        const auto now = std::chrono::steady_clock::now();
        acc[phase] += std::chrono::duration<double>(now - t).count();
        t = now;
    }
};
// events around one step of a chunk generator: [e0, e1) charged to phase a, [e1, e2) to b
struct EventSplit {
    cudaEvent_t e[3] = {};
    EventSplit() { for (auto& v : e) MX_CUDA(cudaEventCreate(&v)); }
    ~EventSplit() { for (auto& v : e) if (v) cudaEventDestroy(v); }
    void rec(int i, cudaStream_t st) { MX_CUDA(cudaEventRecord(e[i], st)); }
    // after the stream is synchronised
    void charge(double* acc, int a, int b) {
        float ms = 0.f;
        MX_CUDA(cudaEventElapsedTime(&ms, e[0], e[1]));
        acc[a] += 1e-3 * ms;
        MX_CUDA(cudaEventElapsedTime(&ms, e[1], e[2]));
        acc[b] += 1e-3 * ms;
    }
};

struct Plan {
    int32_t n = 0, m = 0, c = 0;
    double build_s[kNumPhases] = {};
    Options opt;
    bool built = false;
    int32_t rank = 0, nranks = 1, device = -1;
    // decomposed path (A = R C A_p with a communicator): set by set_comm / set_comm_local, also
    // at nranks = 1 (a one-rank communicator runs every exchange step against itself)
    bool dist = false;
    // shard probe (memxct_plan_set_shard): this device builds rank `rank`'s A_p, A_p^T and
    // exchange maps of a P-way decomposition alone, with no peers and no communicator; the
    // collective steps of the build are replaced by local re-tracing (exchange.cu)
    bool shard = false;
    int32_t tile_tomo = 0, tile_sino = 0;
    bool fused_dot = true;   // CG dots in the SpMV epilogue (MEMXCT_FUSED_DOT=0: separate kernels)
    int32_t part_rows = 0, buffer_entries = 0;  // resolved tuning of A_p (A_p^T: back.R / back.B)
    int32_t ray_block = -1;                     // resolved MEMXCT_OPT_RAY_BLOCK (-1: Hilbert rows)
    int32_t stage_order = -1;                   // resolved MEMXCT_OPT_STAGE_ORDER (-1 Hilbert, 1 slab)

    // domain decomposition: this rank owns Hilbert pixels [t0, t1) and rays [s0, s1)
    std::unique_ptr<Comm> comm;
    std::shared_ptr<LocalGroup> local_group;
    std::vector<uint8_t> unique_id;
    std::string host_comm;  // memxct_plan_set_comm_host: shared-memory segment name
    int64_t t0 = 0, t1 = 0, s0 = 0, s1 = 0;
    std::vector<int64_t> tomo_bounds, sino_bounds;      // per rank, Hilbert index ranges
    std::vector<int64_t> tomo_tile_off, sino_tile_off;  // Hilbert offset of every tile (+ total)
    int64_t nfp = 0;                                    // footprint rays (rows of A_p)
    DevArr<int32_t> fp_rays;                            // their Hilbert ray indices (P > 1)
    Exchange ex;
    SirtState sirt;

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
    int32_t scal_slices = 0, cg_slices = 0;
    // multi-slice SpMM input, slice-interleaved ([ncols][k] fp32, spmm_f32): sized once for the
    // largest slice group the stage buffers admit (ensure_spmm_scratch), so captured graphs never
    // see it move
    DevBuf spmm_xi;
    // staging for *_host calls
    DevBuf h_in, h_out;
    // captured CG solves, keyed on (y, x, iters * 64 + slices, stream); least recently used evicted
    // beyond kMaxGraphs
    std::map<std::tuple<const void*, void*, int32_t, cudaStream_t>, std::unique_ptr<CgGraph>> graphs;
    int64_t graph_clock = 0;
    // buffers replaced by grow() (common.h): kept until destroy, never freed while peers may spin
    std::vector<DevBuf> retired;

    int64_t local_len(int domain) const { return domain == 0 ? t1 - t0 : s1 - s0; }
    int64_t device_bytes() const;
};

// hilbert.cu
void build_hilbert(int32_t h, int32_t w, int32_t t, int32_t* nat_of_h, int32_t* h_of_nat,
                   std::vector<int64_t>* tile_off, cudaStream_t st);
int32_t default_tile(int32_t h, int32_t w);

// trace.cu: Siddon passes over rows [r0, r0 + nrows) (absolute row r = Hilbert ray hray[r], or r
// if hray is null); with `filter`, only segments in Hilbert pixels [lo, hi) count.
//   count: row_len[r - r0];  emit: cols = pixel - lo, row_ids = r (row_ptr chunk-local);
//   hist: atomicAdd(hist[pixel - lo], 1) (lo = 0 without filter)
void trace_count(const Plan& P, const Geometry& G, const int32_t* hray, int64_t r0, int64_t nrows, int64_t lo,
                 int64_t hi, bool filter, int32_t* row_len, cudaStream_t st);
void trace_emit(const Plan& P, const Geometry& G, const int32_t* hray, int64_t r0, int64_t nrows, int64_t lo,
                int64_t hi, const int64_t* row_ptr, uint32_t* cols, float* vals, uint32_t* row_ids,
                cudaStream_t st);
void trace_hist(const Plan& P, const Geometry& G, const int32_t* hray, int64_t r0, int64_t nrows, int64_t lo,
                int64_t hi, bool filter, int32_t* hist, cudaStream_t st);

// rle.cu: block-record encoding of a built layout's stage maps (Layout::rle); returns false (and
// leaves the layout alone) when the encoding does not apply (input indices >= 2^27)
bool encode_map_runs(Layout& L, cudaStream_t st);
bool rle_requested();

// layout.cu: chunked device build of both directions' staged jagged-SELL layouts
void build_matrices(Plan& P, cudaStream_t st);
void widen_i32_to_i64(const int32_t* in, int64_t* out, int64_t n, cudaStream_t st);
void exclusive_scan_i64(const int64_t* in, int64_t* out, int64_t n, cudaStream_t st);
void stable_sort_by_key(const uint32_t* keys_in, uint32_t* keys_out, uint32_t* perm_out, int64_t n,
                        int64_t key_range, cudaStream_t st);
void row_ptr_from_sorted(const uint32_t* row_ids, int64_t nnz, int64_t nrows, int64_t* row_ptr, cudaStream_t st);

// exchange.cu: domain decomposition and the A = R C A_p operators
std::vector<int64_t> partition_ranges(const std::vector<int64_t>& w, int32_t parts);
void decompose(Plan& P, const Geometry& G, cudaStream_t st);
int64_t footprint(Plan& P, const Geometry& G, DevArr<int32_t>& fp_len, cudaStream_t st);
void shard_receive_maps(Plan& P, const Geometry& G, cudaStream_t st);
void build_exchange(Plan& P, cudaStream_t st);
// dot_out (nullable, P > 1): the CG dot of this rank's output part, fused into the last kernel
void apply_forward(Plan& P, const void* x, void* y, cudaStream_t st, double* dot_out = nullptr);
void apply_back(Plan& P, const void* y, void* x, cudaStream_t st, double* dot_out = nullptr,
                bool prepacked = false);
// CG at P > 1 with the sparse collective exchange: the R^T pack of the back projection is fused
// into the x / r update (cg.cu), which scatters every updated owned ray r[i] to its pack positions
// (the reduction map R lists them: {j : recv_idx[j] = i}); apply_back(..., prepacked) then
// starts at the all-to-allv.  Destinations: recv_buf, and this rank's own slice in place.
struct PackTargets {
    const int64_t* red_ptr = nullptr;
    const int32_t* red_pos = nullptr;
    void* rb = nullptr;        // receive / pack buffer
    void* self = nullptr;      // y_fp + sdispl[me]
    int64_t lo = 0, hi = 0;    // pack positions of the own slice: [rdispl[me], rdispl[me + 1])
};
bool cg_fused_pack(const Plan& P);  // the sparse collective path (not dense, not peer)
PackTargets pack_targets(Plan& P);
void time_exchange(Plan& P, int reps, double* us_fwd, double* us_back, cudaStream_t st);
void time_spmv(Plan& P, int reps, double* us_fwd, double* us_back, cudaStream_t st);
double read_ceiling_gbs(int64_t bytes, int reps, cudaStream_t st);  // memxct_read_ceiling
void export_coo(const Layout& L, int32_t* rows, int32_t* cols, float* vals, cudaStream_t st);  // memxct_export_coo
// R (+ CG dot; pa.fold: folded arrival wait and credits, peer.cu) on the shared reduction grid
void reduce_partials(Plan& P, const float* recv, float* y, double* dot_out, const PeerArgs& pa, cudaStream_t st);
void preload_exchange_kernels();
// peer.cu: fused SpMV + exchange over peer memory (EXCHANGE = 1)
void peer_setup(Plan& P, cudaStream_t st);
// dot_out (nullable): <y, y> (forward) / <x, x> (back) of this rank's part, fused into the kernels
void peer_forward(Plan& P, const float* x, float* y, double* dot_out, cudaStream_t st);
void peer_back(Plan& P, const float* y, float* x, double* dot_out, cudaStream_t st);
// v[s * stride] (s < K) summed over ranks in rank order, in place, over peer memory
void peer_allreduce(Plan& P, double* v, int K, int64_t stride, cudaStream_t st);
// K slices, slice-major [K][local_len] fp32 vectors
void apply_forward_batch(Plan& P, int K, const float* x, float* y, cudaStream_t st);
void apply_back_batch(Plan& P, int K, const float* y, float* x, cudaStream_t st);
// allocates the batched-call buffers for the largest slice group; call outside graph capture
// (a no-op under capture); clears the captured solves when a buffer moves
void prepare_batch_scratch(Plan& P, cudaStream_t st);

// spmv.cu
void spmv_init();
// [c0, c1): the CTAs (launch-order positions, Layout::part_order) to run; c1 < 0 = all.  A
// fused dot needs the whole launch.
void spmv_f32(const Layout& L, const float* x, float* y, double* dot_part, double* dot_out,
              unsigned int* ticket, cudaStream_t st, int64_t c0 = 0, int64_t c1 = -1);
void spmv_f64(const Layout& L, const double* x, double* y, double* dot_part, double* dot_out,
              unsigned int* ticket, bool canonical, cudaStream_t st, int64_t c0 = 0, int64_t c1 = -1);
void spmv_f32_remote(const Layout& L, const float* x, const PeerArgs& pa, cudaStream_t st);
// A_p^T of the fused exchange: the footprint input was stored by the owners (peer.cu); with
// pa.fold the kernel waits for their arrival flags and its last CTA returns the credits
void spmv_f32_peer_back(const Layout& L, const float* x, float* y, double* dot_part, double* dot_out,
                        unsigned int* dot_ticket, const PeerArgs& pa, cudaStream_t st);
// K in {1, 2, 4, 8} slices at once: x[s*ldx + i], y[s*ldy + r].  k > 1: x is first interleaved
// into xi ([L.ncols][k], >= L.ncols * k floats) so that the stage gather fetches one slice group
// per map entry with a single 8/16/32 B load
void spmm_f32(const Layout& L, int k, const float* x, int64_t ldx, float* y, int64_t ldy, float* xi,
              cudaStream_t st);
int spmm_max_slices(const Layout& L);

inline void spmv_any(Plan&, const Layout& L, const float* in, float* out, cudaStream_t st) {
    spmv_f32(L, in, out, nullptr, nullptr, nullptr, st);
}
inline void spmv_any(Plan&, const Layout& L, const double* in, double* out, cudaStream_t st) {
    spmv_f64(L, in, out, nullptr, nullptr, nullptr, false, st);
}

// cg.cu
void cg_run(Plan& P, const void* y, void* x, int32_t iters, int32_t slices, cudaStream_t st);
void cg_fetch_norms(Plan& P, int32_t iters, int32_t slices, double* out, cudaStream_t st);

// sirt.cu
void sirt_run(Plan& P, const void* y, void* x, int32_t iters, double* residual_norms, cudaStream_t st);

}  // namespace mx
