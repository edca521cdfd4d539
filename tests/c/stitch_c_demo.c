/*
 * A plain-C consumer of the C ABI (include/stitch.h): no Python, no torch.  Crops an n x m grid
 * of overlapping 256x192 uint16 tiles with known offsets out of one smooth random scene, runs
 * steps 1-7 through stitch_init / stitch_load_grid / stitch_compute_translations (library-owned
 * workspace and stream) and checks every west / north translation against the known offsets,
 * then the bounded mode (stitch_config.pool_tiles) and the error path of a bad tile size.
 * Exit status 0 on success.  Build: gcc -I include stitch_c_demo.c -L<pkg> -lstitch_b200.
 */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "stitch.h"

enum { N = 4, M = 5, H = 192, W = 256, SX = 230, SY = 172 };

static uint32_t lcg(uint32_t* s) { return *s = *s * 1664525u + 1013904223u; }

int main(int argc, char** argv) {
    /* scene: random bumps + per-pixel texture, big enough for every tile */
    const int GW = M * SX + W + 64, GH = N * SY + H + 64;
    float* scene = (float*)calloc((size_t)GW * GH, sizeof(float));
    uint32_t s = 12345u;
    for (int k = 0; k < 4000; ++k) {
        const int cx = (int)(lcg(&s) % (uint32_t)GW), cy = (int)(lcg(&s) % (uint32_t)GH);
        const float a = 200.0f + (float)(lcg(&s) % 3000u), r = 3.0f + (float)(lcg(&s) % 20u);
        for (int y = cy - 3 * (int)r; y <= cy + 3 * (int)r; ++y)
            for (int x = cx - 3 * (int)r; x <= cx + 3 * (int)r; ++x)
                if (x >= 0 && y >= 0 && x < GW && y < GH)
                    scene[(size_t)y * GW + x] +=
                        a * expf(-((float)((x - cx) * (x - cx) + (y - cy) * (y - cy))) / (2 * r * r));
    }
    for (size_t i = 0; i < (size_t)GW * GH; ++i) scene[i] += (float)(lcg(&s) >> 21);   /* texture */
    int ox[N][M], oy[N][M], jx[M], jy[N];
    for (int c = 0; c < M; ++c) jx[c] = (int)(lcg(&s) % 9u);
    for (int r = 0; r < N; ++r) jy[r] = (int)(lcg(&s) % 9u);
    uint16_t* tiles = (uint16_t*)malloc(sizeof(uint16_t) * N * M * H * W);
    for (int r = 0; r < N; ++r)
        for (int c = 0; c < M; ++c) {
            /* perpendicular offsets >= 0: the four candidates of Fig. 2 cover dx, dy >= 0 */
            ox[r][c] = c * SX + jx[c] + r * (1 + c % 2);
            oy[r][c] = r * SY + jy[r] + c * (1 + r % 3);
            uint16_t* t = tiles + ((size_t)r * M + c) * H * W;
            for (int y = 0; y < H; ++y)
                for (int x = 0; x < W; ++x) {
                    float v = 1000.0f + scene[(size_t)(oy[r][c] + y) * GW + ox[r][c] + x] +
                              (float)(lcg(&s) % 41u) - 20.0f;
                    t[y * W + x] = (uint16_t)(v < 0 ? 0 : v > 65535 ? 65535 : v);
                }
        }
    if (argc > 1) {   /* dump the tiles and the known offsets, do not run */
        FILE* f = fopen(argv[1], "wb");
        if (!f) return 1;
        fwrite(tiles, sizeof(uint16_t), (size_t)N * M * H * W, f);
        fwrite(ox, sizeof(int), N * M, f);
        fwrite(oy, sizeof(int), N * M, f);
        fclose(f);
        return 0;
    }
    stitch_config cfg;
    memset(&cfg, 0, sizeof(cfg));
    cfg.tile_width = W;
    cfg.tile_height = H;
    cfg.grid_rows = N;
    cfg.grid_cols = M;
    stitch_ctx* ctx = NULL;
    stitch_status st = stitch_init(&cfg, &ctx);
    if (st != STITCH_OK) {
        printf("stitch_init: %s\n", stitch_status_string(st));
        return 1;
    }
    stitch_pair west[N * M], north[N * M];
    const size_t bytes = sizeof(uint16_t) * N * M * H * W;
    if ((st = stitch_load_grid(ctx, tiles, bytes)) != STITCH_OK ||
        (st = stitch_compute_translations(ctx, west, north)) != STITCH_OK) {
        printf("compute: %s (%s)\n", stitch_status_string(st), stitch_last_error(ctx));
        return 1;
    }
    int bad = 0;
    for (int r = 0; r < N; ++r)
        for (int c = 0; c < M; ++c) {
            const stitch_pair* w = &west[r * M + c];
            const stitch_pair* no = &north[r * M + c];
            if (c > 0 && (w->dx != ox[r][c] - ox[r][c - 1] || w->dy != oy[r][c] - oy[r][c - 1] ||
                          !(w->ccf > 0.9)))
                ++bad;
            if (r > 0 && (no->dx != ox[r][c] - ox[r - 1][c] || no->dy != oy[r][c] - oy[r - 1][c] ||
                          !(no->ccf > 0.9)))
                ++bad;
            if ((c == 0 && w->candidate != 0) || (r == 0 && no->candidate != 0)) ++bad;
        }
    int64_t launches = 0, ffts = 0, pairs = 0;
    stitch_last_counts(ctx, &launches, &ffts, &pairs);
    stitch_destroy(ctx);
    /* the bounded mode: 8 tile slots for 20 tiles, tiles streamed from the host buffer */
    cfg.pool_tiles = 8;
    cfg.chunk_tiles = 2;
    cfg.chunk_pairs = 3;
    stitch_pair w2[N * M], n2[N * M];
    if ((st = stitch_init(&cfg, &ctx)) != STITCH_OK ||
        (st = stitch_compute_translations_from_host_async(ctx, tiles, 0, N * M)) != STITCH_OK ||
        (st = stitch_get_translations(ctx, w2, n2)) != STITCH_OK) {
        printf("bounded mode: %s\n", stitch_status_string(st));
        return 1;
    }
    stitch_destroy(ctx);
    if (memcmp(w2, west, sizeof(west)) != 0 || memcmp(n2, north, sizeof(north)) != 0) ++bad;
    /* a tile size without a compiled plan */
    cfg.tile_height = 191;
    if (stitch_init(&cfg, &ctx) != STITCH_ERR_UNSUPPORTED || ctx != NULL) ++bad;
    printf("C ABI demo: %lld pairs, %lld forward transforms, %lld launches, %d mismatches\n",
           (long long)pairs, (long long)ffts, (long long)launches, bad);
    free(tiles);
    free(scene);
    return bad ? 2 : 0;
}
