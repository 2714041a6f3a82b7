// api.cu -- the C ABI of include/memxct.h.  Argument checking, plan state, error mapping;
// every arithmetic step is delegated to the CUDA kernels of hilbert.cu, trace.cu, layout.cu,
// spmv.cu and cg.cu.  No C++ exception crosses this boundary.
#include <atomic>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "plan.h"

struct memxct_plan {
    mx::Plan P;
};

struct memxct_group {
    std::shared_ptr<mx::LocalGroup> g;
};

namespace mx {

static std::atomic<int64_t> g_launches{0};
void count_launch(int64_t n) { g_launches.fetch_add(n, std::memory_order_relaxed); }
int64_t launch_count() { return g_launches.load(std::memory_order_relaxed); }

int num_sms() {
    static std::mutex mu;
    static std::vector<int> cache;
    int dev = 0;
    MX_CUDA(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(mu);
    if ((int)cache.size() <= dev) cache.resize(dev + 1, 0);
    if (!cache[dev]) MX_CUDA(cudaDeviceGetAttribute(&cache[dev], cudaDevAttrMultiProcessorCount, dev));
    return cache[dev];
}

int64_t Plan::device_bytes() const {
    return fwd.device_bytes() + back.device_bytes() +
           (int64_t)(tomo_nat_of_h.buf.bytes() + tomo_h_of_nat.buf.bytes() + sino_nat_of_h.buf.bytes() +
                     sino_h_of_nat.buf.bytes() + cg_r.bytes() + cg_q.bytes() + cg_s.bytes() + cg_p.bytes() +
                     cg_ax.bytes() + part_fwd.buf.bytes() + part_back.buf.bytes() + part_vec.buf.bytes() +
                     scal.buf.bytes() + tickets.buf.bytes() + h_in.bytes() + h_out.bytes() +
                     fp_rays.buf.bytes() + spmm_xi.bytes()) +
           [this] { int64_t b = 0; for (const DevBuf& r : retired) b += (int64_t)r.bytes(); return b; }() +
           ex.device_bytes();
}

}  // namespace mx

namespace {

thread_local std::string g_last_error;

template <class F> memxct_status_t guarded(F&& f) {
    try {
        f();
        g_last_error.clear();
        return MEMXCT_OK;
    } catch (const mx::Error& e) {
        g_last_error = e.what();
        return e.status;
    } catch (const std::bad_alloc&) {
        g_last_error = "host allocation failed";
        return MEMXCT_ERR_OUT_OF_MEMORY;
    } catch (const std::exception& e) {
        g_last_error = e.what();
        return MEMXCT_ERR_CUDA;
    } catch (...) {
        g_last_error = "unknown error";
        return MEMXCT_ERR_CUDA;
    }
}

mx::Plan& plan_of(memxct_plan_t plan) {
    if (!plan) mx::fail(MEMXCT_ERR_INVALID_ARG, "plan is NULL");
    return plan->P;
}

mx::Plan& built_plan(memxct_plan_t plan) {
    mx::Plan& P = plan_of(plan);
    if (!P.built) mx::fail(MEMXCT_ERR_STATE, "plan used before memxct_build");
    if (P.device >= 0) MX_CUDA(cudaSetDevice(P.device));
    if (P.dist) {  // errors of earlier asynchronous work: NCCL, or a peer wait that gave up
        if (P.comm) P.comm->check_async();
        if (P.ex.peer) mx::check_peer_abort();
    }
    return P;
}

// a plan whose forward/back operators are whole: not a shard probe (which has no peers to
// exchange partials with)
mx::Plan& full_plan(memxct_plan_t plan) {
    mx::Plan& P = built_plan(plan);
    if (P.shard) mx::fail(MEMXCT_ERR_UNSUPPORTED, "a shard probe has no peers: use the memxct_footprint_* calls");
    return P;
}

// a decomposed plan (P >= 1 ranks: NCCL, virtual ranks or a shard probe)
mx::Plan& decomposed_plan(memxct_plan_t plan) {
    mx::Plan& P = built_plan(plan);
    if (!P.dist) mx::fail(MEMXCT_ERR_INVALID_ARG, "the plan is not decomposed (no set_comm / set_shard)");
    return P;
}

cudaStream_t stream_of(void* s) { return reinterpret_cast<cudaStream_t>(s); }

void need(const void* p, const char* what) {
    if (!p) mx::fail(MEMXCT_ERR_INVALID_ARG, std::string(what) + " is NULL");
}

void run_forward(mx::Plan& P, const void* x, void* y, cudaStream_t st) { mx::apply_forward(P, x, y, st); }

void run_back(mx::Plan& P, const void* y, void* x, cudaStream_t st) { mx::apply_back(P, y, x, st); }

void ensure_host_staging(mx::Plan& P) {
    if (!P.h_in.get()) {
        const int64_t mx_len = std::max(P.local_len(0), P.local_len(1));
        P.h_in.alloc(P.esize * std::max<int64_t>(mx_len, 1));
        P.h_out.alloc(P.esize * std::max<int64_t>(mx_len, 1));
    }
}

}  // namespace

extern "C" {

memxct_status_t memxct_plan_create(int32_t n, int32_t projections, int32_t channels, memxct_plan_t* out) {
    return guarded([&] {
        need(out, "out");
        *out = nullptr;
        if (n < 1 || projections < 1 || channels < 1)
            mx::fail(MEMXCT_ERR_INVALID_ARG, "n, projections and channels must be >= 1");
        if ((int64_t)n * n >= ((int64_t)1 << 31) || (int64_t)projections * channels >= ((int64_t)1 << 31))
            mx::fail(MEMXCT_ERR_INVALID_ARG, "n*n and projections*channels must be < 2^31");
        auto* p = new memxct_plan();
        p->P.n = n;
        p->P.m = projections;
        p->P.c = channels;
        *out = p;
    });
}

memxct_status_t memxct_plan_set_option(memxct_plan_t plan, memxct_option_t option, int64_t value) {
    return guarded([&] {
        mx::Plan& P = plan_of(plan);
        if (P.built) mx::fail(MEMXCT_ERR_STATE, "options must be set before memxct_build");
        auto range = [&](int64_t lo, int64_t hi) {
            if (value < lo || value > hi)
                mx::fail(MEMXCT_ERR_INVALID_ARG, "option value out of range [" + std::to_string(lo) + ", " +
                                                     std::to_string(hi) + "]");
        };
        switch (option) {
            case MEMXCT_OPT_TILE_TOMO:
            case MEMXCT_OPT_TILE_SINO:
                range(0, 128);
                if (value != 0 && (value & (value - 1))) mx::fail(MEMXCT_ERR_INVALID_ARG, "tile side must be a power of two");
                (option == MEMXCT_OPT_TILE_TOMO ? P.opt.tile_tomo : P.opt.tile_sino) = value;
                break;
            case MEMXCT_OPT_PART_ROWS:
                range(0, 1024);
                if (value % 32) mx::fail(MEMXCT_ERR_INVALID_ARG, "PART_ROWS must be 0 (auto) or a multiple of 32");
                P.opt.part_rows = value;
                break;
            case MEMXCT_OPT_BUFFER_ENTRIES:
                if (value != 0) range(256, 57344);
                P.opt.buffer_entries = value;
                break;
            case MEMXCT_OPT_PRECISION: range(0, 1); P.opt.precision = value; break;
            case MEMXCT_OPT_CANONICAL: range(0, 1); P.opt.canonical = value; break;
            case MEMXCT_OPT_CG_VARIANT: range(0, 1); P.opt.cg_variant = value; break;
            case MEMXCT_OPT_VECTOR_ORDER: range(0, 1); P.opt.vector_order = value; break;
            case MEMXCT_OPT_SLICES: range(1, 8); P.opt.slices = value; break;
            case MEMXCT_OPT_EXCHANGE: range(0, 2); P.opt.exchange = value; break;
            case MEMXCT_OPT_RAY_BLOCK:
                range(-1, 32);
                if (value > 0 && (value & (value - 1))) mx::fail(MEMXCT_ERR_INVALID_ARG, "RAY_BLOCK must be -1, 0 or a power of two");
                P.opt.ray_block = value;
                break;
            case MEMXCT_OPT_STAGE_ORDER:
                range(-1, 1);
                P.opt.stage_order = value;
                break;
            default: mx::fail(MEMXCT_ERR_INVALID_ARG, "unknown option");
        }
    });
}

memxct_status_t memxct_plan_get_option(memxct_plan_t plan, memxct_option_t option, int64_t* value) {
    return guarded([&] {
        mx::Plan& P = plan_of(plan);
        need(value, "value");
        switch (option) {
            case MEMXCT_OPT_TILE_TOMO: *value = P.built ? P.tile_tomo : P.opt.tile_tomo; break;
            case MEMXCT_OPT_TILE_SINO: *value = P.built ? P.tile_sino : P.opt.tile_sino; break;
            case MEMXCT_OPT_PART_ROWS: *value = P.built ? P.part_rows : P.opt.part_rows; break;
            case MEMXCT_OPT_BUFFER_ENTRIES: *value = P.built ? P.buffer_entries : P.opt.buffer_entries; break;
            case MEMXCT_OPT_PRECISION: *value = P.opt.precision; break;
            case MEMXCT_OPT_CANONICAL: *value = P.opt.canonical; break;
            case MEMXCT_OPT_CG_VARIANT: *value = P.opt.cg_variant; break;
            case MEMXCT_OPT_VECTOR_ORDER: *value = P.opt.vector_order; break;
            case MEMXCT_OPT_SLICES: *value = P.opt.slices; break;
            case MEMXCT_OPT_EXCHANGE: *value = P.opt.exchange; break;
            case MEMXCT_OPT_RAY_BLOCK: *value = P.built ? P.ray_block : P.opt.ray_block; break;
            case MEMXCT_OPT_STAGE_ORDER: *value = P.built ? P.stage_order : P.opt.stage_order; break;
            default: mx::fail(MEMXCT_ERR_INVALID_ARG, "unknown option");
        }
    });
}

memxct_status_t memxct_plan_set_comm(memxct_plan_t plan, int32_t rank, int32_t nranks,
                                     const void* nccl_unique_id, int32_t cuda_device) {
    return guarded([&] {
        mx::Plan& P = plan_of(plan);
        if (P.built) mx::fail(MEMXCT_ERR_STATE, "set_comm must precede memxct_build");
        if (nranks < 1 || rank < 0 || rank >= nranks) mx::fail(MEMXCT_ERR_INVALID_ARG, "bad rank / nranks");
        if (nranks > 1) need(nccl_unique_id, "nccl_unique_id");
        P.unique_id.clear();
        if (nccl_unique_id)
            P.unique_id.assign((const uint8_t*)nccl_unique_id, (const uint8_t*)nccl_unique_id + 128);
        P.rank = rank;
        P.nranks = nranks;
        P.dist = nccl_unique_id != nullptr;
        P.shard = false;
        P.device = cuda_device;
        P.local_group.reset();
        P.host_comm.clear();
    });
}

memxct_status_t memxct_plan_set_comm_host(memxct_plan_t plan, int32_t rank, int32_t nranks, const char* name,
                                          int32_t cuda_device) {
    return guarded([&] {
        mx::Plan& P = plan_of(plan);
        if (P.built) mx::fail(MEMXCT_ERR_STATE, "set_comm must precede memxct_build");
        if (nranks < 1 || nranks > 16 || rank < 0 || rank >= nranks) mx::fail(MEMXCT_ERR_INVALID_ARG, "bad rank / nranks");
        need(name, "name");
        if (name[0] != '/' || std::strlen(name) < 2 || std::strlen(name) > 200 || std::strchr(name + 1, '/'))
            mx::fail(MEMXCT_ERR_INVALID_ARG, "name must be \"/<token>\" (a POSIX shared-memory name)");
        P.unique_id.clear();
        P.local_group.reset();
        P.host_comm = name;
        P.rank = rank;
        P.nranks = nranks;
        P.dist = true;
        P.shard = false;
        P.device = cuda_device;
    });
}

memxct_status_t memxct_host_comm_probe(const char* name, int32_t rank, int32_t nranks, int64_t value,
                                       int64_t* gathered) {
    return guarded([&] {
        need(name, "name");
        need(gathered, "gathered");
        if (nranks < 1 || nranks > 16 || rank < 0 || rank >= nranks) mx::fail(MEMXCT_ERR_INVALID_ARG, "bad rank / nranks");
        if (name[0] != '/' || std::strlen(name) < 2 || std::strlen(name) > 200 || std::strchr(name + 1, '/'))
            mx::fail(MEMXCT_ERR_INVALID_ARG, "name must be \"/<token>\" (a POSIX shared-memory name)");
        const auto v = mx::host_comm_probe(name, rank, nranks, value);
        for (int q = 0; q < nranks; ++q) gathered[q] = v[q];
    });
}

memxct_status_t memxct_plan_set_shard(memxct_plan_t plan, int32_t rank, int32_t nranks, int32_t cuda_device) {
    return guarded([&] {
        mx::Plan& P = plan_of(plan);
        if (P.built) mx::fail(MEMXCT_ERR_STATE, "set_shard must precede memxct_build");
        if (nranks < 1 || rank < 0 || rank >= nranks) mx::fail(MEMXCT_ERR_INVALID_ARG, "bad rank / nranks");
        P.unique_id.clear();
        P.local_group.reset();
        P.host_comm.clear();
        P.rank = rank;
        P.nranks = nranks;
        P.dist = true;
        P.shard = true;
        P.device = cuda_device;
    });
}

memxct_status_t memxct_get_unique_id(void* out) {
    return guarded([&] {
        need(out, "out");
        mx::nccl_unique_id(out);
    });
}

memxct_status_t memxct_local_group_create(int32_t nranks, memxct_group_t* out) {
    return guarded([&] {
        need(out, "out");
        if (nranks < 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "nranks < 1");
        *out = new memxct_group{std::make_shared<mx::LocalGroup>(nranks)};
    });
}

memxct_status_t memxct_local_group_destroy(memxct_group_t group) {
    return guarded([&] { delete group; });
}

memxct_status_t memxct_plan_set_comm_local(memxct_plan_t plan, memxct_group_t group, int32_t rank) {
    return guarded([&] {
        mx::Plan& P = plan_of(plan);
        need(group, "group");
        if (P.built) mx::fail(MEMXCT_ERR_STATE, "set_comm must precede memxct_build");
        if (rank < 0 || rank >= group->g->nranks) mx::fail(MEMXCT_ERR_INVALID_ARG, "bad rank");
        P.rank = rank;
        P.nranks = group->g->nranks;
        P.dist = true;
        P.shard = false;
        P.local_group = group->g;
        P.host_comm.clear();
    });
}

memxct_status_t memxct_partition_ranges(const int64_t* weights, int64_t count, int32_t parts, int64_t* bounds) {
    return guarded([&] {
        need(bounds, "bounds");
        if (count < 0 || parts < 1 || (count > 0 && !weights)) mx::fail(MEMXCT_ERR_INVALID_ARG, "bad arguments");
        std::vector<int64_t> w(weights, weights + count);
        for (int64_t v : w)
            if (v < 0) mx::fail(MEMXCT_ERR_INVALID_ARG, "negative weight");
        const auto b = mx::partition_ranges(w, parts);
        for (int32_t g = 0; g <= parts; ++g) bounds[g] = b[g];
    });
}

memxct_status_t memxct_domain_ranges(memxct_plan_t plan, int32_t domain, int64_t* bounds) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        need(bounds, "bounds");
        if (domain != 0 && domain != 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "domain must be 0 or 1");
        const auto& b = domain == 0 ? P.tomo_bounds : P.sino_bounds;
        for (size_t g = 0; g < b.size(); ++g) bounds[g] = b[g];
    });
}

memxct_status_t memxct_exchange_info(memxct_plan_t plan, int64_t* footprint_rays, int64_t* sent_entries,
                                     int64_t* received_entries, int32_t* peers) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        int64_t sent = 0, np = 0;
        for (int q = 0; q < (int)P.ex.scount.size(); ++q)
            if (q != P.rank) {
                sent += P.ex.scount[q];
                np += (P.ex.scount[q] > 0 || P.ex.rcount[q] > 0);
            }
        int64_t recv = 0;
        for (int q = 0; q < (int)P.ex.rcount.size(); ++q)
            if (q != P.rank) recv += P.ex.rcount[q];
        if (footprint_rays) *footprint_rays = P.nfp;
        if (sent_entries) *sent_entries = sent;
        if (received_entries) *received_entries = recv;
        if (peers) *peers = (int32_t)np;
    });
}

memxct_status_t memxct_build_phases(memxct_plan_t plan, double* seconds) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        need(seconds, "seconds");
        static_assert(mx::kNumPhases == MEMXCT_BUILD_PHASES, "phase table");
        for (int i = 0; i < mx::kNumPhases; ++i) seconds[i] = P.build_s[i];
    });
}

memxct_status_t memxct_build(memxct_plan_t plan, void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = plan_of(plan);
        if (P.built) mx::fail(MEMXCT_ERR_STATE, "plan already built");
        if (P.opt.canonical && P.opt.precision != 1)
            mx::fail(MEMXCT_ERR_INVALID_ARG, "CANONICAL requires PRECISION = MIXED");
        if (P.opt.vector_order == 0 && P.dist)
            mx::fail(MEMXCT_ERR_INVALID_ARG, "natural vector order requires the undecomposed plan");
        int ndev = 0;
        if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
            cudaGetLastError();
            mx::fail(MEMXCT_ERR_CUDA, "no CUDA device: libmemxct has no CPU fallback");
        }
        if (P.device >= 0) MX_CUDA(cudaSetDevice(P.device));
        else MX_CUDA(cudaGetDevice(&P.device));
        mx::spmv_init();
        cudaStream_t st = stream_of(cuda_stream);
        for (double& v : P.build_s) v = 0.0;
        mx::PhaseClock clk(P.build_s, st);
        const auto t_build = clk.t;
        P.tile_tomo = (int32_t)(P.opt.tile_tomo ? P.opt.tile_tomo : mx::default_tile(P.n, P.n));
        P.tile_sino = (int32_t)(P.opt.tile_sino ? P.opt.tile_sino : mx::default_tile(P.m, P.c));
        const int64_t npix = (int64_t)P.n * P.n, nrays = (int64_t)P.m * P.c;
        P.tomo_nat_of_h.alloc(npix);
        P.tomo_h_of_nat.alloc(npix);
        P.sino_nat_of_h.alloc(nrays);
        P.sino_h_of_nat.alloc(nrays);
        mx::build_hilbert(P.n, P.n, P.tile_tomo, P.tomo_nat_of_h.p(), P.tomo_h_of_nat.p(), &P.tomo_tile_off, st);
        mx::build_hilbert(P.m, P.c, P.tile_sino, P.sino_nat_of_h.p(), P.sino_h_of_nat.p(), &P.sino_tile_off, st);
        clk.mark(mx::kPhHilbert);
        P.esize = P.opt.precision == 1 ? 8 : 4;
        if (P.dist) {
            if (P.opt.canonical) mx::fail(MEMXCT_ERR_UNSUPPORTED, "CANONICAL mode is single-GPU only");
            if (P.shard && P.opt.exchange == 1) mx::fail(MEMXCT_ERR_UNSUPPORTED, "a shard probe has no peers to map");
            if (P.shard) P.comm.reset();
            else if (P.local_group) P.comm = mx::make_local_comm(P.local_group, P.rank);
            else if (!P.host_comm.empty()) P.comm = mx::make_host_comm(P.host_comm, P.rank, P.nranks);
            else P.comm = mx::make_nccl_comm(P.rank, P.nranks, P.unique_id.data());
        }
        // CG dots fused into the SpMV epilogue (per-CTA tree + last-CTA sum, deterministic):
        // default since the jagged kernel (3.874 vs 3.882 ms per cfg3 iteration, one kernel
        // fewer per SpMV); MEMXCT_FUSED_DOT=0 restores the separate dot kernels
        const char* fd = std::getenv("MEMXCT_FUSED_DOT");
        P.fused_dot = !(fd && fd[0] == '0');
        mx::build_matrices(P, st);
        MX_CUDA(cudaStreamSynchronize(st));
        P.build_s[mx::kPhTotal] =
            std::chrono::duration<double>(std::chrono::steady_clock::now() - t_build).count();
        P.built = true;
    });
}

memxct_status_t memxct_local_size(memxct_plan_t plan, int32_t domain, int64_t* count) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        need(count, "count");
        if (domain != 0 && domain != 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "domain must be 0 or 1");
        *count = P.local_len(domain);
    });
}

memxct_status_t memxct_local_indices(memxct_plan_t plan, int32_t domain, int64_t* natural_idx) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        need(natural_idx, "natural_idx");
        if (domain != 0 && domain != 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "domain must be 0 or 1");
        const mx::DevArr<int32_t>& a = domain == 0 ? P.tomo_nat_of_h : P.sino_nat_of_h;
        const int64_t lo = domain == 0 ? P.t0 : P.s0, cnt = P.local_len(domain);
        std::vector<int32_t> h(cnt);
        if (cnt > 0) MX_CUDA(cudaMemcpy(h.data(), a.p() + lo, 4 * cnt, cudaMemcpyDeviceToHost));
        for (int64_t i = 0; i < cnt; ++i) natural_idx[i] = h[i];
    });
}

memxct_status_t memxct_forward(memxct_plan_t plan, const void* x_tomo, void* y_sino, void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_tomo, "x_tomo");
        need(y_sino, "y_sino");
        run_forward(P, x_tomo, y_sino, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_back(memxct_plan_t plan, const void* y_sino, void* x_tomo, void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_tomo, "x_tomo");
        need(y_sino, "y_sino");
        run_back(P, y_sino, x_tomo, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_cg(memxct_plan_t plan, const void* y_sino, void* x_tomo, int32_t iters,
                          double* residual_norms, void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_tomo, "x_tomo");
        need(y_sino, "y_sino");
        if (iters < 0) mx::fail(MEMXCT_ERR_INVALID_ARG, "iters < 0");
        cudaStream_t st = stream_of(cuda_stream);
        mx::cg_run(P, y_sino, x_tomo, iters, 1, st);
        if (residual_norms) mx::cg_fetch_norms(P, iters, 1, residual_norms, st);
    });
}

memxct_status_t memxct_forward_host(memxct_plan_t plan, const void* x_host, void* y_host, void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_host, "x_host");
        need(y_host, "y_host");
        ensure_host_staging(P);
        cudaStream_t st = stream_of(cuda_stream);
        MX_CUDA(cudaMemcpyAsync(P.h_in.get(), x_host, P.esize * P.local_len(0), cudaMemcpyHostToDevice, st));
        run_forward(P, P.h_in.get(), P.h_out.get(), st);
        MX_CUDA(cudaMemcpyAsync(y_host, P.h_out.get(), P.esize * P.local_len(1), cudaMemcpyDeviceToHost, st));
        MX_CUDA(cudaStreamSynchronize(st));
    });
}

memxct_status_t memxct_back_host(memxct_plan_t plan, const void* y_host, void* x_host, void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_host, "x_host");
        need(y_host, "y_host");
        ensure_host_staging(P);
        cudaStream_t st = stream_of(cuda_stream);
        MX_CUDA(cudaMemcpyAsync(P.h_in.get(), y_host, P.esize * P.local_len(1), cudaMemcpyHostToDevice, st));
        run_back(P, P.h_in.get(), P.h_out.get(), st);
        MX_CUDA(cudaMemcpyAsync(x_host, P.h_out.get(), P.esize * P.local_len(0), cudaMemcpyDeviceToHost, st));
        MX_CUDA(cudaStreamSynchronize(st));
    });
}

memxct_status_t memxct_cg_host(memxct_plan_t plan, const void* y_host, void* x_host, int32_t iters,
                               double* residual_norms, void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_host, "x_host");
        need(y_host, "y_host");
        if (iters < 0) mx::fail(MEMXCT_ERR_INVALID_ARG, "iters < 0");
        ensure_host_staging(P);
        cudaStream_t st = stream_of(cuda_stream);
        MX_CUDA(cudaMemcpyAsync(P.h_in.get(), y_host, P.esize * P.local_len(1), cudaMemcpyHostToDevice, st));
        mx::cg_run(P, P.h_in.get(), P.h_out.get(), iters, 1, st);
        MX_CUDA(cudaMemcpyAsync(x_host, P.h_out.get(), P.esize * P.local_len(0), cudaMemcpyDeviceToHost, st));
        if (residual_norms) mx::cg_fetch_norms(P, iters, 1, residual_norms, st);
        MX_CUDA(cudaStreamSynchronize(st));
    });
}

memxct_status_t memxct_sirt(memxct_plan_t plan, const void* y_sino, void* x_tomo, int32_t iters,
                            double* residual_norms, void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_tomo, "x_tomo");
        need(y_sino, "y_sino");
        if (iters < 0) mx::fail(MEMXCT_ERR_INVALID_ARG, "iters < 0");
        mx::sirt_run(P, y_sino, x_tomo, iters, residual_norms, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_exchange_time(memxct_plan_t plan, int32_t reps, double* us_forward, double* us_back,
                                     void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(us_forward, "us_forward");
        need(us_back, "us_back");
        mx::time_exchange(P, reps, us_forward, us_back, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_spmv_time(memxct_plan_t plan, int32_t reps, double* us_forward, double* us_back,
                                 void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        need(us_forward, "us_forward");
        need(us_back, "us_back");
        if (reps < 0) mx::fail(MEMXCT_ERR_INVALID_ARG, "reps < 0");
        mx::time_spmv(P, reps, us_forward, us_back, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_read_ceiling(int64_t bytes, int32_t reps, double* gbs, void* cuda_stream) {
    return guarded([&] {
        need(gbs, "gbs");
        *gbs = mx::read_ceiling_gbs(bytes, reps, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_forward_batch(memxct_plan_t plan, int32_t slices, const void* x_tomo, void* y_sino,
                                     void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_tomo, "x_tomo");
        need(y_sino, "y_sino");
        if (slices < 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "slices < 1");
        if (P.esize != 4) mx::fail(MEMXCT_ERR_UNSUPPORTED, "batched projections are FP32 only");
        mx::apply_forward_batch(P, slices, (const float*)x_tomo, (float*)y_sino, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_back_batch(memxct_plan_t plan, int32_t slices, const void* y_sino, void* x_tomo,
                                  void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_tomo, "x_tomo");
        need(y_sino, "y_sino");
        if (slices < 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "slices < 1");
        if (P.esize != 4) mx::fail(MEMXCT_ERR_UNSUPPORTED, "batched projections are FP32 only");
        mx::apply_back_batch(P, slices, (const float*)y_sino, (float*)x_tomo, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_cg_batch(memxct_plan_t plan, int32_t slices, const void* y_sino, void* x_tomo,
                                int32_t iters, double* residual_norms, void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = full_plan(plan);
        need(x_tomo, "x_tomo");
        need(y_sino, "y_sino");
        if (iters < 0) mx::fail(MEMXCT_ERR_INVALID_ARG, "iters < 0");
        if (slices < 1 || slices > 32) mx::fail(MEMXCT_ERR_INVALID_ARG, "slices must be in [1, 32]");
        if (slices > 1 && P.esize != 4) mx::fail(MEMXCT_ERR_UNSUPPORTED, "multi-slice CG is FP32 only");
        cudaStream_t st = stream_of(cuda_stream);
        mx::cg_run(P, y_sino, x_tomo, iters, slices, st);
        if (residual_norms) mx::cg_fetch_norms(P, iters, slices, residual_norms, st);
    });
}

memxct_status_t memxct_footprint_rays(memxct_plan_t plan, int64_t* natural_ray) {
    return guarded([&] {
        mx::Plan& P = decomposed_plan(plan);
        need(natural_ray, "natural_ray");
        std::vector<int32_t> h(P.nfp);
        if (P.nfp > 0) {
            MX_CUDA(cudaMemcpy(h.data(), P.fp_rays.p(), 4 * P.nfp, cudaMemcpyDeviceToHost));
            std::vector<int32_t> perm((size_t)P.m * P.c);
            MX_CUDA(cudaMemcpy(perm.data(), P.sino_nat_of_h.p(), 4 * perm.size(), cudaMemcpyDeviceToHost));
            for (int64_t i = 0; i < P.nfp; ++i) natural_ray[i] = perm[h[i]];
        }
    });
}

memxct_status_t memxct_footprint_forward(memxct_plan_t plan, const void* x_local, void* y_footprint,
                                         void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = decomposed_plan(plan);
        need(x_local, "x_local");
        need(y_footprint, "y_footprint");
        if (P.esize == 4) mx::spmv_any(P, P.fwd, (const float*)x_local, (float*)y_footprint, stream_of(cuda_stream));
        else mx::spmv_any(P, P.fwd, (const double*)x_local, (double*)y_footprint, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_footprint_back(memxct_plan_t plan, const void* y_footprint, void* x_local,
                                      void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = decomposed_plan(plan);
        need(x_local, "x_local");
        need(y_footprint, "y_footprint");
        if (P.esize == 4) mx::spmv_any(P, P.back, (const float*)y_footprint, (float*)x_local, stream_of(cuda_stream));
        else mx::spmv_any(P, P.back, (const double*)y_footprint, (double*)x_local, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_exchange_counts(memxct_plan_t plan, int64_t* send_counts, int64_t* recv_counts) {
    return guarded([&] {
        mx::Plan& P = decomposed_plan(plan);
        for (int q = 0; q < P.nranks; ++q) {
            if (send_counts) send_counts[q] = P.ex.scount[q];
            if (recv_counts) recv_counts[q] = P.ex.rcount[q];
        }
    });
}

memxct_status_t memxct_stats(memxct_plan_t plan, int64_t* nnz, int64_t* stored_slots, int64_t* map_entries,
                             int64_t* device_bytes) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        if (nnz) *nnz = P.fwd.nnz;
        if (stored_slots) *stored_slots = P.fwd.nslots + P.back.nslots;
        if (map_entries) *map_entries = P.fwd.nmap + P.back.nmap;
        if (device_bytes) *device_bytes = P.device_bytes();
    });
}

memxct_status_t memxct_layout_info(memxct_plan_t plan, int32_t dir, int64_t* parts, int64_t* stages,
                                   int64_t* slots, int64_t* map_entries, int64_t* rows, int64_t* nnz,
                                   int64_t* part_rows, int64_t* buffer_entries) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        if (dir != 0 && dir != 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "dir must be 0 or 1");
        const mx::Layout& L = dir == 0 ? P.fwd : P.back;
        if (parts) *parts = L.nparts;
        if (stages) *stages = L.nstages;
        if (slots) *slots = L.nslots;
        if (map_entries) *map_entries = L.nmap;
        if (rows) *rows = L.nrows;
        if (nnz) *nnz = L.nnz;
        if (part_rows) *part_rows = L.R;
        if (buffer_entries) *buffer_entries = L.B;
    });
}

memxct_status_t memxct_layout_export(memxct_plan_t plan, int32_t dir, int64_t p0, int64_t p1,
                                     int64_t* stage_base, int64_t* map_off, int32_t* map, int64_t* slot_off,
                                     uint16_t* ind, float* val, uint16_t* lane_chunks, int64_t* part_row0,
                                     int64_t* n_map, int64_t* n_slot_off, int64_t* n_slots) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        if (dir != 0 && dir != 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "dir must be 0 or 1");
        const mx::Layout& L = dir == 0 ? P.fwd : P.back;
        if (p0 < 0 || p1 > L.nparts || p0 > p1) mx::fail(MEMXCT_ERR_INVALID_ARG, "bad partition range");
        int64_t sb[2], mo[2];
        MX_CUDA(cudaMemcpy(&sb[0], L.stage_base.p() + p0, 8, cudaMemcpyDeviceToHost));
        MX_CUDA(cudaMemcpy(&sb[1], L.stage_base.p() + p1, 8, cudaMemcpyDeviceToHost));
        MX_CUDA(cudaMemcpy(&mo[0], L.map_off.p() + p0, 8, cudaMemcpyDeviceToHost));
        MX_CUDA(cudaMemcpy(&mo[1], L.map_off.p() + p1, 8, cudaMemcpyDeviceToHost));
        const int64_t b0 = sb[0] * L.SPP, b1 = sb[1] * L.SPP;
        int64_t so[2];
        MX_CUDA(cudaMemcpy(&so[0], L.slot_off.p() + b0, 8, cudaMemcpyDeviceToHost));
        MX_CUDA(cudaMemcpy(&so[1], L.slot_off.p() + b1, 8, cudaMemcpyDeviceToHost));
        if (n_map) *n_map = mo[1] - mo[0];
        if (n_slot_off) *n_slot_off = b1 - b0 + 1;
        if (n_slots) *n_slots = so[1] - so[0];
        if (stage_base) MX_CUDA(cudaMemcpy(stage_base, L.stage_base.p() + p0, 8 * (p1 - p0 + 1), cudaMemcpyDeviceToHost));
        if (map_off) MX_CUDA(cudaMemcpy(map_off, L.map_off.p() + p0, 8 * (p1 - p0 + 1), cudaMemcpyDeviceToHost));
        if (map && mo[1] > mo[0]) MX_CUDA(cudaMemcpy(map, L.map.p() + mo[0], 4 * (mo[1] - mo[0]), cudaMemcpyDeviceToHost));
        if (slot_off) MX_CUDA(cudaMemcpy(slot_off, L.slot_off.p() + b0, 8 * (b1 - b0 + 1), cudaMemcpyDeviceToHost));
        if (ind && so[1] > so[0]) MX_CUDA(cudaMemcpy(ind, L.ind.p() + so[0], 2 * (so[1] - so[0]), cudaMemcpyDeviceToHost));
        if (val && so[1] > so[0]) MX_CUDA(cudaMemcpy(val, L.val.p() + so[0], 4 * (so[1] - so[0]), cudaMemcpyDeviceToHost));
        if (part_row0) MX_CUDA(cudaMemcpy(part_row0, L.prow0.p() + p0, 8 * (p1 - p0 + 1), cudaMemcpyDeviceToHost));
        if (lane_chunks && b1 > b0)
            MX_CUDA(cudaMemcpy(lane_chunks, L.lane_chunks.p() + b0 * 32, 2 * 32 * (b1 - b0), cudaMemcpyDeviceToHost));
    });
}

memxct_status_t memxct_export_coo(memxct_plan_t plan, int32_t dir, int32_t* rows, int32_t* cols, float* vals,
                                  void* cuda_stream) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        if (dir != 0 && dir != 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "dir must be 0 or 1");
        need(rows, "rows");
        need(cols, "cols");
        need(vals, "vals");
        mx::export_coo(dir == 0 ? P.fwd : P.back, rows, cols, vals, stream_of(cuda_stream));
    });
}

memxct_status_t memxct_layout_rows(memxct_plan_t plan, int32_t dir, int64_t* out_index) {
    return guarded([&] {
        mx::Plan& P = built_plan(plan);
        need(out_index, "out_index");
        if (dir != 0 && dir != 1) mx::fail(MEMXCT_ERR_INVALID_ARG, "dir must be 0 or 1");
        const mx::Layout& L = dir == 0 ? P.fwd : P.back;
        if (L.out_idx.p()) {
            std::vector<int32_t> h(L.nrows);
            if (L.nrows > 0) MX_CUDA(cudaMemcpy(h.data(), L.out_idx.p(), 4 * L.nrows, cudaMemcpyDeviceToHost));
            for (int64_t r = 0; r < L.nrows; ++r) out_index[r] = h[r];
        } else {
            for (int64_t r = 0; r < L.nrows; ++r) out_index[r] = r;
        }
    });
}

memxct_status_t memxct_plan_destroy(memxct_plan_t plan) {
    if (!plan) return MEMXCT_OK;
    return guarded([&] {
        if (plan->P.device >= 0) cudaSetDevice(plan->P.device);
        delete plan;
    });
}

const char* memxct_status_string(memxct_status_t s) {
    switch (s) {
        case MEMXCT_OK: return "MEMXCT_OK";
        case MEMXCT_ERR_INVALID_ARG: return "MEMXCT_ERR_INVALID_ARG";
        case MEMXCT_ERR_STATE: return "MEMXCT_ERR_STATE";
        case MEMXCT_ERR_OUT_OF_MEMORY: return "MEMXCT_ERR_OUT_OF_MEMORY";
        case MEMXCT_ERR_CUDA: return "MEMXCT_ERR_CUDA";
        case MEMXCT_ERR_NCCL: return "MEMXCT_ERR_NCCL";
        case MEMXCT_ERR_UNSUPPORTED: return "MEMXCT_ERR_UNSUPPORTED";
    }
    return "MEMXCT_ERR_UNKNOWN";
}

const char* memxct_last_error(void) { return g_last_error.c_str(); }

int64_t memxct_kernel_launch_count(void) { return mx::launch_count(); }

}  // extern "C"
