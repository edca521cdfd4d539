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
// result is deterministic without atomics.
#include <cuda_runtime.h>

#include <algorithm>
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

__global__ void compose_overlay(const uint16_t* __restrict__ tiles, const int64_t* __restrict__ pos,
                                int n, int m, int H, int W, int K, int64_t cw, int64_t ch,
                                uint16_t* __restrict__ canvas) {
    constexpr int MAXL = COMPOSE_MAXK + COMPOSE_MAXK * (2 * COMPOSE_MAXK + 1);
    __shared__ int lx[MAXL], ly[MAXL];   // later tiles' origins relative to this tile
    __shared__ int nl;
    const int t = blockIdx.y;
    const int r = t / m, c = t % m;
    const int64_t x0 = pos[2 * (size_t)t], y0 = pos[2 * (size_t)t + 1];
    if (threadIdx.x == 0) {
        int k = 0;
        for (int rr = r; rr <= r + K && rr < n; ++rr)
            for (int cc = (rr == r ? c + 1 : c - K); cc <= c + K; ++cc) {
                if (cc < 0 || cc >= m) continue;
                const size_t u = (size_t)rr * m + cc;
                const int64_t ox = pos[2 * u] - x0, oy = pos[2 * u + 1] - y0;
                if (ox > -W && ox < W && oy > -H && oy < H && k < MAXL) {
                    lx[k] = (int)ox;
                    ly[k] = (int)oy;
                    ++k;
                }
            }
        nl = k;
    }
    __syncthreads();
    const uint16_t* src = tiles + (size_t)t * H * W;
    for (int y = blockIdx.x; y < H; y += gridDim.x) {
        const int64_t Y = y0 + y;
        if (Y < 0 || Y >= ch) continue;
        // x-intervals [a, b) of this row covered by later tiles (tile-local coordinates)
        int a[MAXL], b[MAXL], ni = 0;
        for (int k = 0; k < nl; ++k)
            if (y >= ly[k] && y < ly[k] + H) {
                a[ni] = lx[k];
                b[ni] = lx[k] + W;
                ++ni;
            }
        uint16_t* dst = canvas + (size_t)Y * cw + x0;
        for (int x = threadIdx.x; x < W; x += blockDim.x) {
            if (x0 + x < 0 || x0 + x >= cw) continue;
            bool covered = false;
            for (int k = 0; k < ni; ++k) covered |= (x >= a[k] && x < b[k]);
            if (!covered) dst[x] = src[(size_t)y * W + x];
        }
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
    compose_overlay<<<dim3(H < 64 ? H : 64, nt), 256, 0, s>>>(dev_tiles, dpos, n, m, H, W, K,
                                                            canvas_w, canvas_h, dev_canvas);
    cudaError_t e = cudaGetLastError();
    cudaFreeAsync(dpos, s);
    if (e != cudaSuccess) return STITCH_ERR_CUDA;
    return cudaStreamSynchronize(s) == cudaSuccess ? STITCH_OK : STITCH_ERR_CUDA;
}

}  // extern "C"
