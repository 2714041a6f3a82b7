// hilbert.cu -- two-level pseudo-Hilbert ordering of an H x W domain (sec. 3.2;
// readings R6-R9 in DESIGN.md).
//
// Level 1 (host, O(#tiles)): the T x T tiles are ordered by the generalized Hilbert curve for
// rectangles (gilbert2d, ref. [20] P:1733-1735) and each tile gets an orientation in D4 so that
// the curve enters at the corner nearest the previous tile's exit and leaves toward the next tile
// ("necessary rotations ... to provide data connectivity among tiles").
// Level 2 (device, O(H*W)): one CTA per tile maps curve position d -> cell with the textbook
// Hilbert curve and the tile's orientation, skipping cells outside the domain; a block scan gives
// the rank of each kept cell.
#include <cub/block/block_scan.cuh>

#include <algorithm>
#include <vector>

#include "plan.h"

namespace mx {

namespace {

struct Frame { int32_t x, y, ax, ay, bx, by; };

inline int32_t sgn(int32_t v) { return (v > 0) - (v < 0); }
inline int32_t fdiv2(int32_t v) { return (v >= 0) ? v / 2 : -((-v + 1) / 2); }  // floor(v / 2)

// Generalized Hilbert curve over a w x h grid of tiles, iterative (explicit stack).
void tile_curve(int32_t w, int32_t h, std::vector<int32_t>& tx, std::vector<int32_t>& ty) {
    tx.clear();
    ty.clear();
    std::vector<Frame> stack;
    stack.push_back(w >= h ? Frame{0, 0, w, 0, 0, h} : Frame{0, 0, 0, h, w, 0});
    while (!stack.empty()) {
        Frame f = stack.back();
        stack.pop_back();
        const int32_t W = std::abs(f.ax + f.ay), H = std::abs(f.bx + f.by);
        const int32_t dax = sgn(f.ax), day = sgn(f.ay), dbx = sgn(f.bx), dby = sgn(f.by);
        if (H == 1 || W == 1) {
            const int32_t cnt = (H == 1) ? W : H;
            const int32_t sx = (H == 1) ? dax : dbx, sy = (H == 1) ? day : dby;
            for (int32_t i = 0; i < cnt; ++i) { tx.push_back(f.x + i * sx); ty.push_back(f.y + i * sy); }
            continue;
        }
        int32_t ax2 = fdiv2(f.ax), ay2 = fdiv2(f.ay), bx2 = fdiv2(f.bx), by2 = fdiv2(f.by);
        const int32_t w2 = std::abs(ax2 + ay2), h2 = std::abs(bx2 + by2);
        if (2 * W > 3 * H) {
            if ((w2 & 1) && W > 2) { ax2 += dax; ay2 += day; }
            // children visited in order: [a-half 1, a-half 2]  -> push reversed
            stack.push_back(Frame{f.x + ax2, f.y + ay2, f.ax - ax2, f.ay - ay2, f.bx, f.by});
            stack.push_back(Frame{f.x, f.y, ax2, ay2, f.bx, f.by});
        } else {
            if ((h2 & 1) && H > 2) { bx2 += dbx; by2 += dby; }
            stack.push_back(Frame{f.x + (f.ax - dax) + (bx2 - dbx), f.y + (f.ay - day) + (by2 - dby),
                                  -bx2, -by2, -(f.ax - ax2), -(f.ay - ay2)});
            stack.push_back(Frame{f.x + bx2, f.y + by2, f.ax, f.ay, f.bx - bx2, f.by - by2});
            stack.push_back(Frame{f.x, f.y, bx2, by2, ax2, ay2});
        }
    }
}

inline int64_t box_dist(int64_t px, int64_t py, int64_t bx, int64_t by, int64_t T) {
    const int64_t x0 = bx * T, x1 = x0 + T - 1, y0 = by * T, y1 = y0 + T - 1;
    const int64_t dx = std::max<int64_t>({0, x0 - px, px - x1});
    const int64_t dy = std::max<int64_t>({0, y0 - py, py - y1});
    return dx + dy;
}

// Textbook Hilbert curve position d -> (x, y) on a T x T grid; starts (0,0), ends (T-1, 0).
__device__ __forceinline__ void hilbert_d2xy(int32_t T, int32_t d, int32_t& x, int32_t& y) {
    int32_t px = 0, py = 0, t = d;
    for (int32_t s = 1; s < T; s <<= 1) {
        const int32_t rx = (t >> 1) & 1;
        const int32_t ry = (t ^ rx) & 1;
        if (!ry) {
            if (rx) { px = s - 1 - px; py = s - 1 - py; }
            const int32_t tmp = px; px = py; py = tmp;
        }
        px += s * rx;
        py += s * ry;
        t >>= 2;
    }
    x = px;
    y = py;
}

constexpr int kHilThreads = 512;
constexpr int kHilItems = 32;  // T <= 128 -> T*T <= 16384 = 512 * 32

__global__ void __launch_bounds__(kHilThreads)
hilbert_cells_kernel(int32_t H, int32_t W, int32_t T, const int32_t* __restrict__ tx,
                     const int32_t* __restrict__ ty, const uint8_t* __restrict__ orient,
                     const int64_t* __restrict__ rank_off, int32_t* __restrict__ nat_of_h,
                     int32_t* __restrict__ h_of_nat) {
    using Scan = cub::BlockScan<int32_t, kHilThreads>;
    __shared__ typename Scan::TempStorage tmp;
    const int32_t k = blockIdx.x;
    const int32_t bx = tx[k] * T, by = ty[k] * T;
    const uint8_t o = orient[k];
    const bool flipx = o & 1, flipy = o & 2, swp = o & 4;
    const int32_t cells = T * T;
    const int32_t per = (cells + kHilThreads - 1) / kHilThreads;  // blocked arrangement
    const bool full = (bx + T <= W) && (by + T <= H);
    int32_t valid = 0;
    // pass 1: count kept cells of this thread's block of d values
    if (!full) {
        for (int32_t q = 0; q < per; ++q) {
            const int32_t d = threadIdx.x * per + q;
            if (d >= cells) break;
            int32_t u, v;
            hilbert_d2xy(T, d, u, v);
            const int32_t uu = swp ? v : u, vv = swp ? u : v;
            const int32_t gx = bx + (flipx ? T - 1 - uu : uu), gy = by + (flipy ? T - 1 - vv : vv);
            valid += (gx < W && gy < H);
        }
    }
    int32_t before = 0;
    if (!full) Scan(tmp).ExclusiveSum(valid, before);
    const int64_t base = rank_off[k];
    for (int32_t q = 0; q < per; ++q) {
        const int32_t d = threadIdx.x * per + q;
        if (d >= cells) break;
        int32_t u, v;
        hilbert_d2xy(T, d, u, v);
        const int32_t uu = swp ? v : u, vv = swp ? u : v;
        const int32_t gx = bx + (flipx ? T - 1 - uu : uu), gy = by + (flipy ? T - 1 - vv : vv);
        if (gx < W && gy < H) {
            const int64_t r = base + (full ? d : before++);
            const int64_t cell = (int64_t)gy * W + gx;
            nat_of_h[r] = (int32_t)cell;
            h_of_nat[cell] = (int32_t)r;
        }
    }
}

}  // namespace

int32_t default_tile(int32_t h, int32_t w) {
    // reading R7: largest power of two T with 8T <= min(H, W), clamped to [4, 64]
    const int32_t mn = std::min(h, w);
    int32_t t = 4;
    while (t * 2 <= 64 && (int64_t)t * 2 * 8 <= mn) t *= 2;
    return t;
}

void build_hilbert(int32_t H, int32_t W, int32_t T, int32_t* nat_of_h, int32_t* h_of_nat,
                   std::vector<int64_t>* tile_off, cudaStream_t st) {
    if (T < 1 || T > 128 || (T & (T - 1))) fail(MEMXCT_ERR_INVALID_ARG, "tile side must be a power of two in [1, 128]");
    const int32_t rt = (H + T - 1) / T, ct = (W + T - 1) / T;
    std::vector<int32_t> tx, ty;
    tile_curve(ct, rt, tx, ty);  // x = tile column, y = tile row
    const int64_t nt = (int64_t)tx.size();
    if (nt != (int64_t)rt * ct) fail(MEMXCT_ERR_CUDA, "internal: tile curve size mismatch");
    std::vector<uint8_t> orient(nt);
    std::vector<int64_t> off(nt);
    int64_t ex = 0, ey = 0, acc = 0;
    for (int64_t k = 0; k < nt; ++k) {
        int64_t nx, ny;  // the tile after k (extrapolated past the last one)
        if (k + 1 < nt) { nx = tx[k + 1]; ny = ty[k + 1]; }
        else if (k > 0) { nx = 2 * (int64_t)tx[k] - tx[k - 1]; ny = 2 * (int64_t)ty[k] - ty[k - 1]; }
        else { nx = tx[k] + 1; ny = ty[k]; }
        // exit corner: along x first, then along y, whichever is nearer the next tile
        const int64_t gx0 = (int64_t)tx[k] * T, gy0 = (int64_t)ty[k] * T;
        const int64_t xa = T - 1 - ex, ya = ey;  // exit differing from entry in x
        const int64_t xb = ex, yb = T - 1 - ey;  // exit differing from entry in y
        const bool use_b = box_dist(gx0 + xb, gy0 + yb, nx, ny, T) < box_dist(gx0 + xa, gy0 + ya, nx, ny, T);
        const int64_t xx = use_b ? xb : xa, xy = use_b ? yb : ya;
        orient[k] = (uint8_t)((ex != 0 ? 1 : 0) | (ey != 0 ? 2 : 0) | (use_b ? 4 : 0));
        off[k] = acc;
        acc += (int64_t)std::min<int64_t>(T, W - gx0) * std::min<int64_t>(T, H - gy0);
        if (k + 1 < nt) {  // entry of the next tile: nearest of its corners in fixed order
            const int64_t gx = gx0 + xx, gy = gy0 + xy;
            const int64_t cx[4] = {0, T - 1, 0, T - 1}, cy[4] = {0, 0, T - 1, T - 1};
            int64_t best = -1;
            for (int q = 0; q < 4; ++q) {
                const int64_t px = (int64_t)tx[k + 1] * T + cx[q], py = (int64_t)ty[k + 1] * T + cy[q];
                const int64_t dd = std::abs(px - gx) + std::abs(py - gy);
                if (best < 0 || dd < best) { best = dd; ex = cx[q]; ey = cy[q]; }
            }
        }
    }
    DevArr<int32_t> dtx, dty;
    DevArr<uint8_t> dor;
    DevArr<int64_t> doff;
    dtx.alloc(nt); dty.alloc(nt); dor.alloc(nt); doff.alloc(nt);
    MX_CUDA(cudaMemcpyAsync(dtx.p(), tx.data(), nt * 4, cudaMemcpyHostToDevice, st));
    MX_CUDA(cudaMemcpyAsync(dty.p(), ty.data(), nt * 4, cudaMemcpyHostToDevice, st));
    MX_CUDA(cudaMemcpyAsync(dor.p(), orient.data(), nt, cudaMemcpyHostToDevice, st));
    MX_CUDA(cudaMemcpyAsync(doff.p(), off.data(), nt * 8, cudaMemcpyHostToDevice, st));
    if (tile_off) {
        *tile_off = off;
        tile_off->push_back(acc);
    }
    hilbert_cells_kernel<<<(unsigned)nt, kHilThreads, 0, st>>>(H, W, T, dtx.p(), dty.p(), dor.p(),
                                                                doff.p(), nat_of_h, h_of_nat);
    MX_LAUNCHED();
    MX_CUDA(cudaStreamSynchronize(st));  // host vectors above go out of scope
}

}  // namespace mx
