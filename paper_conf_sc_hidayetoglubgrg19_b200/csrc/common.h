// common.h -- internal error handling, device buffers and launch accounting for libmemxct.
#pragma once

#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <cstdlib>

#include <cstdint>
#include <cstdio>
#include <stdexcept>
#include <string>
#include <utility>
#include <vector>

#include "memxct.h"

namespace mx {

// Internal exception; converted to a memxct_status_t at the C ABI boundary (api.cu).
struct Error : std::runtime_error {
    memxct_status_t status;
    Error(memxct_status_t s, const std::string& m) : std::runtime_error(m), status(s) {}
};

[[noreturn]] inline void fail(memxct_status_t s, const std::string& m) { throw Error(s, m); }

inline void cuda_check(cudaError_t e, const char* what, const char* file, int line) {
    if (e != cudaSuccess) {
        memxct_status_t s = (e == cudaErrorMemoryAllocation) ? MEMXCT_ERR_OUT_OF_MEMORY : MEMXCT_ERR_CUDA;
        if (e == cudaErrorMemoryAllocation) cudaGetLastError();  // clear the sticky-free error
        fail(s, std::string(what) + ": " + cudaGetErrorString(e) + " (" + file + ":" +
                    std::to_string(line) + ")");
    }
}
#define MX_CUDA(call) ::mx::cuda_check((call), #call, __FILE__, __LINE__)
// After every kernel launch: launch-configuration errors surface here.
#define MX_LAUNCHED() do { ::mx::count_launch(); MX_CUDA(cudaGetLastError()); } while (0)

void count_launch(int64_t n = 1);
int64_t launch_count();

// MEMXCT_ALLOC_TRACE=1: report every cudaMalloc / cudaFree slower than 20 ms on stderr
// (diagnostic of the build-time variance)
inline std::chrono::steady_clock::time_point trace_clock() { return std::chrono::steady_clock::now(); }
inline void trace_slow(const char* what, size_t bytes, std::chrono::steady_clock::time_point t0) {
    static const bool on = [] {
        const char* e = std::getenv("MEMXCT_ALLOC_TRACE");
        return e && e[0] == '1';
    }();
    if (!on) return;
    const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    if (ms > 20.0) fprintf(stderr, "[memxct] %s(%zu B) %.1f ms\n", what, bytes, ms);
}

// Owning device allocation (cudaMalloc); freed on destruction, so an OOM in the middle of a
// build leaves the plan destroyable.
class DevBuf {
public:
    DevBuf() = default;
    explicit DevBuf(size_t bytes) { alloc(bytes); }
    DevBuf(const DevBuf&) = delete;
    DevBuf& operator=(const DevBuf&) = delete;
    DevBuf(DevBuf&& o) noexcept : p_(o.p_), n_(o.n_) { o.p_ = nullptr; o.n_ = 0; }
    DevBuf& operator=(DevBuf&& o) noexcept {
        if (this != &o) { reset(); p_ = o.p_; n_ = o.n_; o.p_ = nullptr; o.n_ = 0; }
        return *this;
    }
    ~DevBuf() { reset(); }
    void alloc(size_t bytes) {
        reset();
        if (bytes == 0) return;
        void* p = nullptr;
        const auto t0 = trace_clock();
        cudaError_t e = cudaMalloc(&p, bytes);
        trace_slow("cudaMalloc", bytes, t0);
        if (e != cudaSuccess) {
            cudaGetLastError();
            fail(e == cudaErrorMemoryAllocation ? MEMXCT_ERR_OUT_OF_MEMORY : MEMXCT_ERR_CUDA,
                 "cudaMalloc(" + std::to_string(bytes) + " B): " + cudaGetErrorString(e));
        }
        p_ = p;
        n_ = bytes;
        g_bytes_ += bytes;
    }
    void reset() {
        if (p_) {
            const auto t0 = trace_clock();
            cudaFree(p_);
            trace_slow("cudaFree", n_, t0);
            g_bytes_ -= n_;
        }
        p_ = nullptr;
        n_ = 0;
    }
    template <class T> T* as() const { return static_cast<T*>(p_); }
    void* get() const { return p_; }
    size_t bytes() const { return n_; }
    static int64_t live_bytes() { return g_bytes_; }

private:
    void* p_ = nullptr;
    size_t n_ = 0;
    static inline int64_t g_bytes_ = 0;
};

template <class T> struct DevArr {
    DevBuf buf;
    int64_t n = 0;
    void alloc(int64_t count) { buf.alloc(sizeof(T) * (size_t)(count > 0 ? count : 0)); n = count; }
    T* p() const { return buf.as<T>(); }
    void reset() { buf.reset(); n = 0; }
};

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Streaming multiprocessors of the current device (148 on B200), for grid sizing.
int num_sms();

// Grow-only reallocation: the previous buffer moves to `retired` (kept until the plan is
// destroyed) instead of being freed.  cudaFree synchronises the whole device, and with the
// fused peer exchange another rank's kernels may be spinning on this rank's next launch; CUDA
// graphs captured against the previous buffer also stay valid.
inline void grow(std::vector<DevBuf>& retired, DevBuf& b, size_t bytes) {
    if (b.bytes() >= bytes) return;
    if (b.get()) retired.push_back(std::move(b));
    b.alloc(bytes);
}
template <class T> inline void grow(std::vector<DevBuf>& retired, DevArr<T>& a, int64_t count) {
    if (a.n >= count && a.p()) return;
    if (a.p()) retired.push_back(std::move(a.buf));
    a.alloc(count);
}

}  // namespace mx
