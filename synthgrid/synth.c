/*
 * synth.c — seeded synthetic tile-grid fixture (INPUT GENERATOR ONLY).
 *
 * Shared by the oracle side (tests) and the CUDA side (tests, bench): it
 * holds none of the method's arithmetic (no transform, no correlation), only
 * a stateless, integer-only procedural "scene" and a crop of it per tile, so
 * every consumer sees bit-identical uint16 tiles for a given seed.
 *
 * Workload shape: grids of 16-bit grayscale
 * 1392x1040 tiles with overlapping neighbours.  The paper's A10 data is not
 * available, so the scene is procedural; DESIGN.md "Input
 * recipe" states the recipe.  Geometry (tile origins) is decided in Python
 * (synthgrid/__init__.py) and passed in; this file only renders pixels.
 *
 * Scene g(X, Y) at global pixel (X, Y) >= 0:
 *   base 30000
 *   + 3 octaves of value noise (cells 128, 32, 8 px; amplitudes 16000, 8000,
 *     4000) with integer smoothstep interpolation of hashed lattice values
 *   + hashed per-pixel scene detail, uniform in [-2000, 2000]
 * Tile pixel = clamp(g(ox + x, oy + y) + read_noise, 0, 65535), read noise
 * = sum of 4 hashed uniforms in [-17, 17] (sigma ~ 20 DN), keyed by the
 * tile id so overlapping tiles differ by independent noise.
 * All arithmetic is 64-bit integer, so results are platform independent.
 */
#include <stdint.h>
#include <stdlib.h>
#include <pthread.h>

static inline uint64_t mix64(uint64_t z) {           /* splitmix64 finaliser */
    z += 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

static inline uint64_t hash3(uint64_t seed, uint64_t a, uint64_t b) {
    return mix64(seed ^ mix64(a ^ mix64(b + 0x632BE59BD9B4E019ULL)));
}

/* cheaper single-round hash for per-pixel streams */
static inline uint64_t hash_px(uint64_t key, uint64_t a, uint64_t b) {
    return mix64(key ^ (a * 0xD6E8FEB86659FD93ULL) ^ (b * 0xA0761D6478BD642FULL));
}

#define N_OCT 3
static const int64_t OCT_LOG2[N_OCT] = {7, 5, 3};          /* cell 128, 32, 8 px */
static const int64_t OCT_AMP[N_OCT] = {16000, 8000, 4000};

/* smoothstep weight of fraction f/S scaled by S^3:  3 f^2 S - 2 f^3 */
static inline int64_t sstep(int64_t f, int64_t S) { return 3 * f * f * S - 2 * f * f * f; }

static inline int64_t lattice(uint64_t seed, int oct, int64_t i, int64_t j) {
    return (int64_t)(hash3(seed + 0x1000u * (uint64_t)(oct + 1), (uint64_t)i, (uint64_t)j) & 0xFFFF);
}

/* Render one tile with origin (ox, oy) into out[H][W]. */
void synth_tile(uint64_t seed, int64_t ox, int64_t oy, int H, int W,
                uint64_t tile_key, uint16_t* out) {
    for (int y = 0; y < H; ++y) {
        const int64_t Y = oy + y;
        /* per-octave row state: lattice row index and y weight */
        int64_t jy[N_OCT], wy[N_OCT], S3[N_OCT];
        const uint64_t kd = mix64(seed ^ 0xD1B54A32D192ED03ULL);
        const uint64_t kn = mix64(seed ^ tile_key ^ 0x8CB92BA72F3D8DD7ULL);
        for (int o = 0; o < N_OCT; ++o) {
            const int64_t S = (int64_t)1 << OCT_LOG2[o];
            jy[o] = Y >> OCT_LOG2[o];
            wy[o] = sstep(Y & (S - 1), S);
            S3[o] = S * S * S;
        }
        int64_t cur_i[N_OCT], L00[N_OCT], L10[N_OCT], L01[N_OCT], L11[N_OCT];
        for (int o = 0; o < N_OCT; ++o) cur_i[o] = INT64_MIN;
        uint16_t* row = out + (size_t)y * (size_t)W;
        for (int x = 0; x < W; ++x) {
            const int64_t X = ox + x;
            int64_t v = 30000;
            for (int o = 0; o < N_OCT; ++o) {
                const int64_t S = (int64_t)1 << OCT_LOG2[o];
                const int64_t i = X >> OCT_LOG2[o];
                if (i != cur_i[o]) {
                    cur_i[o] = i;
                    L00[o] = lattice(seed, o, i, jy[o]);
                    L10[o] = lattice(seed, o, i + 1, jy[o]);
                    L01[o] = lattice(seed, o, i, jy[o] + 1);
                    L11[o] = lattice(seed, o, i + 1, jy[o] + 1);
                }
                const int64_t wx = sstep(X & (S - 1), S);
                /* bilinear blend in S^3 fixed point, one axis at a time */
                const int64_t top = L00[o] * (S3[o] - wx) + L10[o] * wx;   /* <= 2^16 * S^3 */
                const int64_t bot = L01[o] * (S3[o] - wx) + L11[o] * wx;
                const int sh = 3 * (int)OCT_LOG2[o];                         /* S^3 = 2^sh */
                const int64_t t = top >> sh, b = bot >> sh;                  /* in [0, 65535] */
                const int64_t val = (t * (S3[o] - wy[o]) + b * wy[o]) >> sh;
                v += ((val - 32768) * OCT_AMP[o]) / 32768;
            }
            const uint64_t hd = hash_px(kd, (uint64_t)X, (uint64_t)Y);
            v += (int64_t)(hd % 4001u) - 2000;
            const uint64_t hn = hash_px(kn, (uint64_t)x, (uint64_t)y);
            int64_t noise = 0;
            for (int q = 0; q < 4; ++q) noise += (int64_t)((hn >> (16 * q)) & 0xFFFF) % 35 - 17;
            v += noise;
            if (v < 0) v = 0;
            if (v > 65535) v = 65535;
            row[x] = (uint16_t)v;
        }
    }
}

/*
 * Low-texture scene ("cells" texture): the paper's
 * sparse early colonies with "few distinguishable features".  A flat background
 * of 2000 DN plus isolated bright cells and nothing else (no value noise, no per-pixel scene
 * detail): lattice cell (i, j) of CELL_G px holds a cell with probability density/65536, at a
 * hashed centre inside it, radius R in [5, 30] px, amplitude A in [3000, 30000] DN, profile
 * A (1 - d^2/R^2)^2 for d < R (a compactly supported, Gaussian-like bump in integer
 * arithmetic).  Per-tile read noise as above.  An overlap without cells correlates noise only.
 */
#define CELL_G 64
static inline int64_t cells_at(uint64_t seed, int64_t X, int64_t Y, uint32_t density) {
    int64_t v = 2000;
    const int64_t ci = X / CELL_G, cj = Y / CELL_G;
    for (int64_t j = cj - 1; j <= cj + 1; ++j) {
        if (j < 0) continue;
        for (int64_t i = ci - 1; i <= ci + 1; ++i) {
            if (i < 0) continue;
            const uint64_t h = hash3(seed ^ 0x5EEDCE11ULL, (uint64_t)i, (uint64_t)j);
            if ((h & 0xFFFF) >= density) continue;
            const int64_t cx = i * CELL_G + (int64_t)((h >> 16) % CELL_G);
            const int64_t cy = j * CELL_G + (int64_t)((h >> 24) % CELL_G);
            const int64_t R = 5 + (int64_t)((h >> 32) % 26);
            const int64_t A = 3000 + (int64_t)((h >> 40) % 27001);
            const int64_t dx = X - cx, dy = Y - cy, d2 = dx * dx + dy * dy, R2 = R * R;
            if (d2 >= R2) continue;
            const int64_t q = R2 - d2;
            v += A * q * q / (R2 * R2);
        }
    }
    return v;
}

void synth_tile_cells(uint64_t seed, int64_t ox, int64_t oy, int H, int W, uint64_t tile_key,
                      uint32_t density, uint16_t* out) {
    const uint64_t kn = mix64(seed ^ tile_key ^ 0x8CB92BA72F3D8DD7ULL);
    for (int y = 0; y < H; ++y) {
        uint16_t* row = out + (size_t)y * (size_t)W;
        for (int x = 0; x < W; ++x) {
            int64_t v = cells_at(seed, ox + x, oy + y, density);
            const uint64_t hn = hash_px(kn, (uint64_t)x, (uint64_t)y);
            for (int q = 0; q < 4; ++q) v += (int64_t)((hn >> (16 * q)) & 0xFFFF) % 35 - 17;
            if (v < 0) v = 0;
            if (v > 65535) v = 65535;
            row[x] = (uint16_t)v;
        }
    }
}

typedef struct {
    uint64_t seed;
    const int64_t* origins;   /* [count][2] = (ox, oy) */
    const uint64_t* keys;     /* [count] */
    int H, W;
    int64_t count;
    uint16_t* out;
    int64_t next;
    pthread_mutex_t mu;
    int texture;          /* 0: value noise + detail (default), 1: sparse cells */
    uint32_t density;     /* cells: lattice-cell occupancy in 1/65536 */
} job_t;

static void* worker(void* p) {
    job_t* j = (job_t*)p;
    for (;;) {
        pthread_mutex_lock(&j->mu);
        const int64_t t = j->next++;
        pthread_mutex_unlock(&j->mu);
        if (t >= j->count) break;
        uint16_t* dst = j->out + (size_t)t * (size_t)j->H * (size_t)j->W;
        if (j->texture == 1)
            synth_tile_cells(j->seed, j->origins[2 * t], j->origins[2 * t + 1], j->H, j->W,
                             j->keys[t], j->density, dst);
        else
            synth_tile(j->seed, j->origins[2 * t], j->origins[2 * t + 1], j->H, j->W, j->keys[t],
                       dst);
    }
    return NULL;
}

/* Render `count` tiles (origins[t] = (ox, oy), keys[t] = noise key) into out[count][H][W]
 * using `threads` POSIX threads; texture 0 = the default scene, 1 = sparse cells at
 * `density` / 65536 per lattice cell.  Returns 0 on success. */
int synth_tiles_tex(uint64_t seed, const int64_t* origins, const uint64_t* keys, int64_t count,
                    int H, int W, int threads, int texture, uint32_t density, uint16_t* out) {
    if (!origins || !keys || !out || H <= 0 || W <= 0 || count < 0) return 1;
    if (texture != 0 && texture != 1) return 1;
    if (threads < 1) threads = 1;
    if (threads > 256) threads = 256;
    job_t j = {seed, origins, keys, H, W, count, out, 0, PTHREAD_MUTEX_INITIALIZER, texture,
               density};
    pthread_t th[256];
    for (int i = 0; i < threads; ++i) pthread_create(&th[i], NULL, worker, &j);
    for (int i = 0; i < threads; ++i) pthread_join(th[i], NULL);
    return 0;
}

int synth_tiles(uint64_t seed, const int64_t* origins, const uint64_t* keys, int64_t count,
                int H, int W, int threads, uint16_t* out) {
    return synth_tiles_tex(seed, origins, keys, count, H, W, threads, 0, 0, out);
}

/* Per-key uniform integer in [0, bound] (used for origin jitter in Python). */
int64_t synth_jitter(uint64_t seed, uint64_t a, uint64_t b, int64_t bound) {
    return (int64_t)(hash3(seed ^ 0xA0761D6478BD642FULL, a, b) % (uint64_t)(bound + 1));
}
