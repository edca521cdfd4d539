// phase23.cu — stitching phases 2 and 3 on top of the phase-1 translations
// (§III).
//
// Phase 2: "resolves the over-constraint in the system and computes absolute
// displacements.  It selects a subset of the relative displacements or uses a global
// optimization approach".  The paper names no algorithm; reading C19: select
// the subset that is a MAXIMUM SPANNING TREE of the tile graph weighted by each pair's CCF
// (the most reliable translations), then absolute positions are path sums from the root
// tile (0, 0) along the tree -- path-invariant by construction.  Host code (a few
// thousand edges; not a hot path).
//
// Phase 3 (Fig. 13 "overlay", L1446): compose the stitched image.  Overlay
// blend: in the overlap of two tiles the later tile (row-major order) is on top.  The GPU
// kernel writes every canvas pixel exactly once -- a tile's pixel is skipped when a later
// tile within K rows/columns covers it (K found on the host from the positions) -- so the
// result is deterministic without atomics.  Each row of a tile writes one clear span with
// 16-byte loads and stores (bandwidth-bound: ~2 x 2 bytes per canvas pixel).
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <climits>
#include <cmath>
#include <numeric>
#include <vector>

#include "../../include/stitch.h"

namespace {

struct Edge {
    int32_t a, b;      // a = neighbour (west/north), b = tile
    int32_t dx, dy;    // origin of b in a's frame
    double w;          // CCF
    int32_t id;
};

int find(std::vector<int32_t>& p, int32_t x) {
    while (p[x] != x) {
        p[x] = p[p[x]];
        x = p[x];
    }
    return x;
}

constexpr int COMPOSE_MAXK = 4;   // later tiles considered: K rows x (2K+1) columns
constexpr int COMPOSE_MAXL = COMPOSE_MAXK + COMPOSE_MAXK * (2 * COMPOSE_MAXK + 1);
constexpr int COMPOSE_WARPS = 8;  // one warp per tile row at a time
constexpr int COMPOSE_ROWB = 8;   // CTAs per tile (rows strided over CTAs and warps)

// 8 pixels starting S pixels (S < 8, warp-uniform) into the 16 pixels of two aligned 16-byte
// segments: the 256-bit pair shifted right by 64, 32 and 16 bits as S's bits say
__device__ __forceinline__ uint4 window8(const uint4& a, const uint4& b, int S) {
    const bool s4 = S & 4, s2 = S & 2;
    const uint32_t w0 = s4 ? a.z : a.x, w1 = s4 ? a.w : a.y, w2 = s4 ? b.x : a.z,
                   w3 = s4 ? b.y : a.w, w4 = s4 ? b.z : b.x, w5 = s4 ? b.w : b.y;
    const uint32_t v0 = s2 ? w1 : w0, v1 = s2 ? w2 : w1, v2 = s2 ? w3 : w2, v3 = s2 ? w4 : w3,
                   v4 = s2 ? w5 : w4;
    const int sh = (S & 1) * 16;
    return make_uint4(__funnelshift_r(v0, v1, sh), __funnelshift_r(v1, v2, sh),
                      __funnelshift_r(v2, v3, sh), __funnelshift_r(v3, v4, sh));
}

// One tile row's canvas span [A, B) (clear of later tiles) in 16-byte-aligned canvas chunks of
// 8 pixels (chunk j = canvas x [8j - e, 8j - e + 8)): lanes take U chunks each at a time
// (loads first, then stores: U chunks in flight); a chunk is two aligned 16-byte source
// segments realigned in registers (S = the row's source misalignment in pixels) and one
// 16-byte store.  The <= 7 pixels before the first and after the last whole chunk go one per
// lane.
__device__ __forceinline__ void compose_span_vec(const uint16_t* __restrict__ src,
                                                 uint16_t* __restrict__ crow, int64_t x0,
                                                 int64_t A, int64_t B, int lane) {
    const int64_t e = (int64_t)(reinterpret_cast<uintptr_t>(crow) / 2 % 8);
    const int64_t jA = (A + e + 7) >> 3, jB = (B + e) >> 3;     // whole chunks [jA, jB)
    if (jA >= jB) {                                             // B - A < 16
        if (A + lane < B) crow[A + lane] = src[A + lane - x0];
        return;
    }
    const int S = (int)(((8 * jA - e - x0) % 8 + 8) % 8);
    constexpr int U = 4;
    for (int64_t jb = jA + lane; jb < jB; jb += 32 * U) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t j = jb + 32 * u;
            if (j < jB) {
                const uint4* s4 = reinterpret_cast<const uint4*>(src + (8 * j - e - x0 - S));
                v[u] = window8(__ldg(s4), S ? __ldg(s4 + 1) : make_uint4(0, 0, 0, 0), S);
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t j = jb + 32 * u;
            if (j < jB) *reinterpret_cast<uint4*>(crow + 8 * j - e) = v[u];
        }
    }
    const int64_t h1 = 8 * jA - e, t0 = 8 * jB - e;             // head [A, h1), tail [t0, B)
    if (lane < 8 && A + lane < h1) crow[A + lane] = src[A + lane - x0];
    if (lane >= 8 && lane < 16 && t0 + lane - 8 < B) crow[t0 + lane - 8] = src[t0 + lane - 8 - x0];
}

template <bool VEC>
__global__ void __launch_bounds__(32 * COMPOSE_WARPS)
    compose_overlay(const uint16_t* __restrict__ tiles, const int64_t* __restrict__ pos, int n,
                    int m, int H, int W, int K, int64_t cw, int64_t ch,
                    uint16_t* __restrict__ canvas) {
    // later tiles within K rows / columns, one per thread: their origins relative to this
    // tile, or ly = INT_MIN / 2 (matches no row) where there is none or it cannot overlap
    __shared__ int lx[COMPOSE_MAXL], ly[COMPOSE_MAXL];
    const int t = blockIdx.y;
    const int r = t / m, c = t % m;
    const int64_t x0 = pos[2 * (size_t)t], y0 = pos[2 * (size_t)t + 1];
    const int nl = K + K * (2 * K + 1);     // (r, c+1..c+K), then rows r+1..r+K, cols c-K..c+K
    if (threadIdx.x < nl) {
        const int i = threadIdx.x;
        const int rr = i < K ? r : r + 1 + (i - K) / (2 * K + 1);
        const int cc = i < K ? c + 1 + i : c - K + (i - K) % (2 * K + 1);
        int ox = 0, oy = INT_MIN / 2;
        if (rr < n && cc >= 0 && cc < m) {
            const size_t u = (size_t)rr * m + cc;
            const int64_t dx = pos[2 * u] - x0, dy = pos[2 * u + 1] - y0;
            if (dx > -W && dx < W && dy > -H && dy < H) {
                ox = (int)dx;
                oy = (int)dy;
            }
        }
        lx[i] = ox;
        ly[i] = oy;
    }
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int y = blockIdx.x * COMPOSE_WARPS + warp; y < H; y += gridDim.x * COMPOSE_WARPS) {
        const int64_t Y = y0 + y;
        if (Y < 0 || Y >= ch) continue;                 // warp-uniform
        // All tiles are W wide, so a later tile's row covers a prefix (its x <= 0) or a suffix
        // of this row: the clear part is one range [P, Sx) of tile-local x.
        int P = 0, Sx = W;
        for (int k = 0; k < nl; ++k)
            if (y >= ly[k] && y < ly[k] + H) {
                if (lx[k] <= 0) P = max(P, lx[k] + W);
                else Sx = min(Sx, lx[k]);
            }
        const int64_t A = max(x0 + P, (int64_t)0), B = min(x0 + Sx, cw);   // canvas x range
        if (A >= B) continue;
        uint16_t* crow = canvas + (size_t)Y * cw;
        const uint16_t* src = tiles + ((size_t)t * H + y) * W;
        if constexpr (VEC)
            compose_span_vec(src, crow, x0, A, B, lane);
        else
            for (int64_t X = A + lane; X < B; X += 32) crow[X] = src[X - x0];
    }
}

}  // namespace

extern "C" {

stitch_status stitch_global_positions(int32_t n, int32_t m, const stitch_pair* west,
                                      const stitch_pair* north, int64_t* pos_xy,
                                      int32_t* parent) {
    if (n < 1 || m < 1 || !west || !north || !pos_xy) return STITCH_ERR_INVALID_ARG;
    const int32_t nt = n * m;
    std::vector<Edge> edges;
    edges.reserve((size_t)2 * nt);
    for (int32_t t = 0; t < nt; ++t) {
        const int32_t r = t / m, c = t % m;
        if (c >= 1 && west[t].candidate > 0 && std::isfinite(west[t].ccf))
            edges.push_back({t - 1, t, west[t].dx, west[t].dy, west[t].ccf, 2 * t});
        if (r >= 1 && north[t].candidate > 0 && std::isfinite(north[t].ccf))
            edges.push_back({t - m, t, north[t].dx, north[t].dy, north[t].ccf, 2 * t + 1});
    }
    // Kruskal, largest CCF first (ties: lower edge id) -- deterministic
    std::sort(edges.begin(), edges.end(), [](const Edge& x, const Edge& y) {
        return x.w != y.w ? x.w > y.w : x.id < y.id;
    });
    std::vector<int32_t> uf(nt);
    std::iota(uf.begin(), uf.end(), 0);
    std::vector<std::vector<int32_t>> adj(nt);   // indices into `tree`
    std::vector<Edge> tree;
    for (const Edge& e : edges) {
        const int32_t ra = find(uf, e.a), rb = find(uf, e.b);
        if (ra == rb) continue;
        uf[ra] = rb;
        adj[e.a].push_back((int32_t)tree.size());
        adj[e.b].push_back((int32_t)tree.size());
        tree.push_back(e);
    }
    // path sums from the root of every component (its smallest tile) along the tree
    std::vector<char> seen(nt, 0);
    std::vector<int32_t> stack;
    for (int32_t root = 0; root < nt; ++root) {
        if (seen[root]) continue;
        seen[root] = 1;
        pos_xy[2 * root] = 0;
        pos_xy[2 * root + 1] = 0;
        if (parent) parent[root] = -1;
        stack.push_back(root);
        while (!stack.empty()) {
            const int32_t u = stack.back();
            stack.pop_back();
            for (const int32_t ei : adj[u]) {
                const Edge& e = tree[ei];
                const int32_t v = e.a == u ? e.b : e.a;
                if (seen[v]) continue;
                seen[v] = 1;
                const int64_t s = e.a == u ? 1 : -1;     // b = a + (dx, dy)
                pos_xy[2 * v] = pos_xy[2 * u] + s * e.dx;
                pos_xy[2 * v + 1] = pos_xy[2 * u + 1] + s * e.dy;
                if (parent) parent[v] = u;
                stack.push_back(v);
            }
        }
    }
    return STITCH_OK;
}

stitch_status stitch_compose_overlay(const uint16_t* dev_tiles, int32_t n, int32_t m, int32_t H,
                                     int32_t W, const int64_t* host_pos_xy, int64_t canvas_w,
                                     int64_t canvas_h, uint16_t* dev_canvas, void* stream) {
    const stitch_status st = stitch_compose_overlay_async(dev_tiles, n, m, H, W, host_pos_xy,
                                                          canvas_w, canvas_h, dev_canvas, stream);
    if (st != STITCH_OK) return st;
    return cudaStreamSynchronize((cudaStream_t)stream) == cudaSuccess ? STITCH_OK : STITCH_ERR_CUDA;
}

stitch_status stitch_compose_overlay_async(const uint16_t* dev_tiles, int32_t n, int32_t m,
                                           int32_t H, int32_t W, const int64_t* host_pos_xy,
                                           int64_t canvas_w, int64_t canvas_h,
                                           uint16_t* dev_canvas, void* stream) {
    nvtxRangePushA("stitch_compose_overlay_async");
    struct Pop {
        ~Pop() { nvtxRangePop(); }
    } pop_;
    if (!dev_tiles || !host_pos_xy || !dev_canvas || n < 1 || m < 1 || H < 1 || W < 1 ||
        canvas_w < 1 || canvas_h < 1)
        return STITCH_ERR_INVALID_ARG;
    const int32_t nt = n * m;
    if (nt > 65535) return STITCH_ERR_UNSUPPORTED;   // one grid row of CTAs per tile
    cudaStream_t s = (cudaStream_t)stream;
    int64_t* dpos = nullptr;
    if (cudaMallocAsync(&dpos, sizeof(int64_t) * 2 * nt, s) != cudaSuccess) return STITCH_ERR_CUDA;
    if (cudaMemcpyAsync(dpos, host_pos_xy, sizeof(int64_t) * 2 * nt, cudaMemcpyHostToDevice, s) !=
        cudaSuccess)
        return STITCH_ERR_CUDA;
    // neighbourhood radius: how many rows / columns apart two overlapping tiles can be
    int K = 1;
    for (int32_t t = 0; t < nt; ++t) {
        const int32_t r = t / m, c = t % m;
        for (int dr = 0; dr <= 8; ++dr)
            for (int dc = -8; dc <= 8; ++dc) {
                const int32_t rr = r + dr, cc = c + dc;
                if ((dr == 0 && dc <= 0) || rr >= n || cc < 0 || cc >= m) continue;
                const int32_t u = rr * m + cc;
                const int64_t ox = host_pos_xy[2 * u] - host_pos_xy[2 * t];
                const int64_t oy = host_pos_xy[2 * u + 1] - host_pos_xy[2 * t + 1];
                if (ox > -W && ox < W && oy > -H && oy < H) K = std::max(K, std::max(dr, std::abs(dc)));
            }
    }
    if (K > COMPOSE_MAXK) return STITCH_ERR_UNSUPPORTED;   // overlaps spanning > 4 tiles
    // 16-byte vector path: tile rows 16-byte aligned and whole 16-byte segments per row (reads
    // never pass the row's end); otherwise pixel by pixel
    const bool vec = W % 8 == 0 && reinterpret_cast<uintptr_t>(dev_tiles) % 16 == 0 &&
                     reinterpret_cast<uintptr_t>(dev_canvas) % 2 == 0;
    const int rb = std::min(COMPOSE_ROWB, (H + COMPOSE_WARPS - 1) / COMPOSE_WARPS);
    if (vec)
        compose_overlay<true><<<dim3(rb, nt), 32 * COMPOSE_WARPS, 0, s>>>(
            dev_tiles, dpos, n, m, H, W, K, canvas_w, canvas_h, dev_canvas);
    else
        compose_overlay<false><<<dim3(rb, nt), 32 * COMPOSE_WARPS, 0, s>>>(
            dev_tiles, dpos, n, m, H, W, K, canvas_w, canvas_h, dev_canvas);
    cudaError_t e = cudaGetLastError();
    cudaFreeAsync(dpos, s);
    return e == cudaSuccess ? STITCH_OK : STITCH_ERR_CUDA;
}

}  // extern "C"
