/*
 * stitch.h — C ABI of the B200-native PCIAM tile-pair translation engine.
 *
 * Computes phase 1 of the stitching method of Blattner et al., ICPP 2014
 * (§III): the relative displacement (translation) of every
 * west and north neighbour pair of a grid of overlapping 16-bit tiles, by
 * Fourier phase correlation (PCIAM, Fig. 1 steps 1-7; Fig. 2
 * pciam(); Fig. 3 ccf(); Fig. 4 grid).
 *
 * Every step runs in hand-written sm_100a CUDA kernels behind this ABI (no
 * cuFFT, no CPU fallback).  Arguments are plain pointers and sizes; no torch
 * or CUDA types appear in the signatures (streams / device memory are passed
 * as void*).  All functions return a stitch_status; no C++ exception crosses
 * the boundary.  On error the contents of output arrays are unspecified and
 * stitch_last_error(ctx) holds a message.
 *
 * Conventions
 *  - Tile layout: uint16 [H][W] row-major, W (x) contiguous.  A grid is
 *    [n][m][H][W]: n tile rows, m tile columns, tile t = r*m + c.
 *  - Pair (A, B) = (west or north neighbour, tile) (reading C1);
 *    the translation (dx, dy) is the origin of B in A's frame, chosen among
 *    the four candidates {x, W-x} x {y, H-y} of the correlation peak
 *    (Fig. 2 l.8-12).
 *  - A context covers the tile range [tile_begin, tile_end) of the grid (a
 *    row band under multi-GPU partitioning) and computes the pairs whose
 *    tile B lies in that range; it also needs the tile row before the range
 *    (the halo, tiles [halo_begin, tile_begin), halo_begin = max(0, tile_begin - m)).
 *  - Every entry point selects the context's device for its duration and
 *    restores the caller's current device before returning.
 *  - A context is not thread-safe.  Work is enqueued on the context's stream
 *    in issue order: device inputs must be complete (ordered before) on that
 *    stream when a call that reads them is made.
 */
#ifndef STITCH_H
#define STITCH_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct stitch_ctx stitch_ctx; /* opaque, owned by the library */

typedef enum {
    STITCH_OK = 0,
    STITCH_ERR_INVALID_ARG = 1, /* null pointer, bad size, bad range, pool too small */
    STITCH_ERR_UNSUPPORTED = 2, /* tile size without a compiled FFT plan; unsupported mode mix */
    STITCH_ERR_OUT_OF_MEMORY = 3,
    STITCH_ERR_CUDA = 4,        /* a CUDA runtime error; see stitch_last_error */
    STITCH_ERR_NCCL = 5,        /* NCCL library missing or an NCCL call failed (multi-rank halo) */
    STITCH_ERR_STATE = 6        /* e.g. compute before load */
} stitch_status;

/* stitch_config.flags */
#define STITCH_FLAG_NO_GRAPH 1u /* launch the step directly instead of replaying a captured CUDA graph */
#define STITCH_FLAG_SERIAL 2u   /* one stream for every kernel (no forward / pair / CCF concurrency) */

typedef struct {
    int32_t tile_width;   /* W (x, contiguous). Compiled plans: 1392x1040, 256x192, 48x40, 58x26 */
    int32_t tile_height;  /* H (y) */
    int32_t grid_rows;    /* n >= 1 */
    int32_t grid_cols;    /* m >= 1 */
    int32_t device;       /* CUDA ordinal */
    int32_t tile_begin;   /* first owned tile (row-major index); 0 for the whole grid */
    int32_t tile_end;     /* one past the last owned tile; 0 => n*m.  With world_size > 1 and both
                             0, the library derives rank's balanced band [rank*n*m/R, (rank+1)*n*m/R) */
    int32_t chunk_pairs;  /* pairs per inverse-transform launch (K3/K4/K5); 0 => default (160) */
    int32_t chunk_tiles;  /* tiles per forward-transform launch (K1/K2); 0 => default (64;
                             pool_tiles/4 in the bounded mode) */
    int32_t precision;    /* arithmetic of steps 2-5: 0 = fp32 (default), 1 = fp64 (the paper's "double
                             complex" transforms; north_star's optional fp64 path).
                             The CCF (steps 6-7) is exact integer moments -> fp64 either way.
                             Anything else -> STITCH_ERR_INVALID_ARG. */
    void* stream;         /* cudaStream_t to enqueue on (e.g. torch's current stream); NULL => library-created */
    void* workspace;      /* caller-owned device memory of >= stitch_workspace_size bytes (e.g. a torch
                             tensor), 256-byte aligned; NULL => the library allocates with cudaMalloc */
    size_t workspace_bytes;
    int32_t pool_tiles;   /* 0 (default): every resident tile keeps its pixels and spectrum in device memory
                             for the whole step.  > 0: BOUNDED mode (the paper's buffer pool with
                             reference counts): a fixed pool of this many tile slots (raw pixels +
                             spectrum each); a slot is recycled once every pair reading its tile (<= 4, Fig. 4)
                             has finished, so device memory no longer grows with the grid.  Tiles come from
                             stitch_compute_translations_from_host_async (copied into slots as they are
                             needed).  fp32 only; INVALID_ARG if the pool cannot hold one tile row plus one
                             forward chunk (about m + chunk_tiles slots); UNSUPPORTED with precision 1 or an
                             NCCL exchange. */
    int32_t rank;         /* this process's rank (0-based) when world_size > 1 */
    int32_t world_size;   /* 0 or 1: single context.  > 1: row-band partition over world_size ranks */
    const void* nccl_id;  /* world_size > 1: the 128-byte ncclUniqueId made by stitch_nccl_unique_id on rank 0
                             and broadcast by the caller (e.g. over torch.distributed).  Then stitch_init joins
                             an NCCL communicator (collective: every rank must call it) and each step moves
                             the halo row's spectra from rank-1 to rank over NCCL send/recv inside the
                             library, overlapped with the interior pairs (SURVEY §8(e), P:L994-998,
                             L1512-1517).  NULL: no communicator; the caller moves the halo
                             (stitch_spectra_range + the split step) or the context recomputes it. */
    uint32_t flags;       /* STITCH_FLAG_* (0 = default: concurrent streams, graph replay) */
} stitch_config;

/*
 * One pair's result (Fig. 2 output "max correlation, x-disp & y-disp", P:L528;
 * Fig. 4 output "2 arrays of tuples ([correlation, x, y])"), 64 bytes.
 */
typedef struct {
    int32_t dx, dy;        /* chosen translation: origin of tile B in tile A's frame */
    double ccf;            /* CCF (Fig. 3) of the chosen candidate; NaN if absent / none valid */
    int32_t candidate;     /* 1..4 in Fig. 2 order (c1..c4); 0 = absent or no valid candidate */
    int32_t peak_x, peak_y;/* argmax of |iFFT2(NCC)| in [0,W) x [0,H) (step 5) */
    float peak;            /* max |iFFT2(NCC)| / (W*H) */
    double ccf_k[4];       /* CCF of each candidate c1..c4 (NaN if invalid: empty region or zero variance) */
} stitch_pair;

/* Static message for a status code. */
const char* stitch_status_string(stitch_status s);

/*
 * Write a new 128-byte NCCL unique id to out128 (ncclGetUniqueId; call on rank 0, broadcast
 * the bytes, pass them as stitch_config.nccl_id on every rank).  NCCL is loaded at run time
 * (libnccl.so.2, e.g. the one torch ships); STITCH_ERR_NCCL if it cannot be loaded or fails.
 */
stitch_status stitch_nccl_unique_id(void* out128);

/* Bytes of device workspace a context with this config needs (for config.workspace). */
stitch_status stitch_workspace_size(const stitch_config* cfg, size_t* bytes);

/* Number of pairs the context computes for this config (Fig. 4 order, tile B in range). */
stitch_status stitch_pair_count(const stitch_config* cfg, int64_t* count);

/*
 * Create a context: validates the config, selects the compiled FFT plan, carves /
 * allocates device memory, uploads twiddle tables, the pair list and (bounded mode) the
 * slot schedule; joins the NCCL communicator if nccl_id is given.
 * Errors: INVALID_ARG (null, n/m < 1, bad tile range or rank, workspace too small, pool too
 * small), UNSUPPORTED (tile size, mode mix), OUT_OF_MEMORY, CUDA, NCCL.  *out is NULL on error.
 */
stitch_status stitch_init(const stitch_config* cfg, stitch_ctx** out);

/*
 * Step 1 (the paper's read + copier stages): copy the
 * tiles this context needs -- [halo_begin, tile_end) -- from the caller's
 * host grid into device memory.  host_grid points at the WHOLE grid
 * [n][m][H][W] (n_bytes = n*m*H*W*2).  Synchronous with respect to the host
 * buffer: it may be reused as soon as the call returns (the call waits for
 * the copy, and so for work enqueued before it on the context stream).
 * Errors: INVALID_ARG (size), STATE (bounded-mode context: tiles arrive with
 * stitch_compute_translations_from_host_async), CUDA.
 */
stitch_status stitch_load_grid(stitch_ctx* ctx, const uint16_t* host_grid, size_t n_bytes);

/*
 * Partial load: `tiles` points at tile `first_tile` of a [count][H][W] run of
 * consecutive row-major tiles that must cover [halo_begin, tile_end) (see
 * stitch_resident_range).  on_device != 0 => device memory (stream-ordered,
 * asynchronous); host memory => synchronous as stitch_load_grid.  Lets each
 * rank of a row-band partition hold only its own rows.
 * Errors: INVALID_ARG if the run does not cover the range; STATE (bounded mode).
 */
stitch_status stitch_load_tiles(stitch_ctx* ctx, const uint16_t* tiles, int32_t first_tile,
                                int32_t count, int32_t on_device);

/* Resident tile range of the context: halo_begin = max(0, tile_begin - m). */
stitch_status stitch_resident_range(stitch_ctx* ctx, int32_t* halo_begin, int32_t* tile_begin,
                                    int32_t* tile_end);

/* Same as stitch_load_grid from device memory (e.g. a torch CUDA tensor holding the whole
 * grid); stream-ordered and asynchronous. */
stitch_status stitch_load_grid_device(stitch_ctx* ctx, const uint16_t* dev_grid, size_t n_bytes);

/*
 * Steps 2-7 for every pair of the range (Fig. 4), results left on the device;
 * asynchronous on the context stream (no host synchronisation).  With an NCCL
 * communicator this includes the halo exchange (rank k sends the spectra of its
 * last tile row to k+1 and receives its halo row from k-1 while its interior
 * pairs run).  Errors: STATE if no grid was loaded (or bounded mode); CUDA; NCCL.
 */
stitch_status stitch_compute_translations_async(stitch_ctx* ctx);

/*
 * Steps 2-7 and copy-out: fills west[t] / north[t] for every owned tile t
 * (arrays of n*m entries indexed by row-major tile index; entries outside
 * the owned range are left untouched; a tile with no west (c = 0) or north
 * (r = 0) neighbour gets candidate 0, ccf NaN).  Synchronous.
 */
stitch_status stitch_compute_translations(stitch_ctx* ctx, stitch_pair* west, stitch_pair* north);

/*
 * Steps 1-7 with step 1 pipelined (the paper's read/copier stages feeding its GPU stages,
 * P:L1030-1040): `tiles` is a HOST run of consecutive tiles starting at `first_tile`
 * covering the resident range (as stitch_load_tiles).  Each forward chunk's tiles are
 * copied host-to-device on their own stream right before that chunk's transforms (into
 * recycled pool slots in the bounded mode), so the copy of later chunks overlaps the
 * transforms and pairs of earlier ones.  Asynchronous: the host buffer must stay valid and
 * unmodified until stitch_get_translations / stitch_synchronize returns.  Pinned
 * (page-locked) memory is needed for the overlap (pageable memory works, without it).
 * fp64 contexts load, then compute.
 * Errors: INVALID_ARG (null pointer, range does not cover the resident tiles); CUDA.
 */
stitch_status stitch_compute_translations_from_host_async(stitch_ctx* ctx, const uint16_t* tiles,
                                                         int32_t first_tile, int32_t count);

/* Copy the results of the last compute to the host (same layout as above). Synchronous. */
stitch_status stitch_get_translations(stitch_ctx* ctx, stitch_pair* west, stitch_pair* north);

/* Forward transforms only (step 2) for all resident tiles; asynchronous. */
stitch_status stitch_forward_async(stitch_ctx* ctx);

/*
 * Split form of a step, for a caller-managed halo exchange:
 *   stitch_forward_range_async -- step 2 for the resident tiles [first_tile, first_tile+count)
 *     (global row-major indices; INVALID_ARG if not resident);
 *   stitch_spectra_range -- device address and size of the resident spectra of a tile range
 *     (Q15 unit phasors F/|F|, u32 [count][H][pitch]; contiguous), so the caller can send the
 *     last tile row of its band to the next rank and receive its halo row instead of
 *     recomputing it;
 *   stitch_pairs_part_async -- steps 3-7 for part of the pairs: 0 all, 1 the INTERIOR pairs
 *     (tile A owned: they need no halo spectrum, so they can run while the halo is in
 *     flight), 2 the BOUNDARY pairs (tile A in the halo).  1 then 2 == 0, bit for bit.
 *   stitch_pairs_async == stitch_pairs_part_async(ctx, 0).
 * compute_translations_async == forward_range_async(all resident) + pairs_async.
 * STATE in the bounded mode.
 */
stitch_status stitch_forward_range_async(stitch_ctx* ctx, int32_t first_tile, int32_t count);
stitch_status stitch_spectra_range(stitch_ctx* ctx, int32_t first_tile, int32_t count,
                                   void** dev_ptr, size_t* bytes);
stitch_status stitch_pairs_async(stitch_ctx* ctx);
stitch_status stitch_pairs_part_async(stitch_ctx* ctx, int32_t part);

/*
 * Test hook: copy tile t's resident half spectrum F(ky, kx), ky in [0,H),
 * kx in [0, W/2] (complex64, [H][W/2+1][2] floats) to the host, recomputed by
 * the context's forward kernels.  Valid after a load.  Synchronous.
 * STATE on an fp64 or bounded-mode context.
 */
stitch_status stitch_debug_spectrum(stitch_ctx* ctx, int32_t tile, float* host_out);

/*
 * Test hook of the fp64 path (precision = 1): tile t's complex
 * half spectrum F(ky, kx) (step 2; "double complex") as
 * [H][W/2+1][2] doubles, recomputed by the same fp64 forward kernels.  The
 * context's resident store holds F/|F| in Q31 fixed point (the only part step 3 uses).
 * Synchronous.  STITCH_ERR_STATE on an fp32 context.
 */
stitch_status stitch_debug_spectrum_f64(stitch_ctx* ctx, int32_t tile, double* host_out);

/*
 * Test hook (reading C11): the normalised correlation surface |iFFT2(NCC)| / (W*H) of one
 * pair (steps 3-4), [H][W] floats row-major, computed by the same K3 + K4
 * transforms the step uses (K4 storing the surface instead of reducing it to its argmax),
 * from the spectra of the last forward transforms.  Pair = (kind 0: west, 1: north) of
 * global tile `tile`.  fp32 resident contexts only (STATE otherwise); INVALID_ARG if the
 * context does not compute that pair.  Synchronous.
 */
stitch_status stitch_debug_surface(stitch_ctx* ctx, int32_t tile, int32_t kind, float* host_out);

/* Wait for all work enqueued on the context stream. */
stitch_status stitch_synchronize(stitch_ctx* ctx);

/*
 * Counters of the last compute: kernel launches issued by the library, and
 * the Table I operation counts: forward transforms, pairs
 * (= NCC products, inverse transforms, max reductions, CCF1..4 evaluations).
 */
stitch_status stitch_last_counts(stitch_ctx* ctx, int64_t* launches, int64_t* forward_ffts,
                                 int64_t* pairs);

/* Device time of the last compute per stage, milliseconds (CUDA events, timing mode 1 or 2):
 * ms[0] forward (K1+K2), ms[1] pair transforms (K3+K4), ms[2] CCF (K5+K6), ms[3] total. */
stitch_status stitch_last_timings(stitch_ctx* ctx, float* ms4);

/* Event timing mode: 0 off (default), 1 per-stage events, 2 per-stage + one event after
 * every kernel launch (for per-kernel durations; one stream, perturbs the timeline
 * slightly), 3 the concurrent schedule launched directly with an event pair around every
 * launch (stitch_timeline).  Anything else: INVALID_ARG. */
stitch_status stitch_set_timing(stitch_ctx* ctx, int enabled);

/* Mode-2 timings of the last compute per kernel K1..K6: summed device ms and launch counts.
 * Valid after stitch_synchronize / stitch_get_translations. */
stitch_status stitch_kernel_timings(stitch_ctx* ctx, float* ms6, int64_t* launches6);

/*
 * Measurement hook: after a compute with stitch_set_timing(ctx, 3) and stitch_synchronize /
 * stitch_get_translations, the launch timeline: kernel id (0..5 = K1..K6), stream (0 forward,
 * 1 pairs, 2 CCF), start and end in ms from the step's start.  Up to `capacity` records are
 * written; *count = the number of records.  STATE if no timeline was collected.
 */
stitch_status stitch_timeline(stitch_ctx* ctx, int32_t* kernel, int32_t* stream, float* start_ms,
                              float* end_ms, int64_t capacity, int64_t* count);

/*
 * Phase 2 (NEXT row f3): absolute tile positions from the phase-1
 * translations.  The paper names no algorithm (reading C19): the translations
 * of a MAXIMUM SPANNING TREE of the tile graph weighted by CCF are kept (Kruskal, ties by
 * pair index) and positions are path sums from the root tile along the tree.
 *   west, north: [n*m] as filled by stitch_compute_translations (candidate 0 = no edge)
 *   pos_xy:      out [n*m][2] (x, y) of each tile's origin; the smallest tile of each
 *                connected component is its origin (0, 0)
 *   parent:      optional out [n*m] tree parent (-1 for a root); may be NULL
 * Host-only (no device work).  Errors: INVALID_ARG.
 */
stitch_status stitch_global_positions(int32_t n, int32_t m, const stitch_pair* west,
                                      const stitch_pair* north, int64_t* pos_xy, int32_t* parent);

/*
 * Phase 3 (NEXT row f4; Fig. 13 overlay L1446): compose the stitched
 * image on the device by overlay blend -- in an overlap the later tile (row-major) is on
 * top; every canvas pixel is written exactly once (deterministic, no atomics).
 *   dev_tiles:  device uint16 [n][m][H][W];  host_pos_xy: [n*m][2] tile origins (canvas px)
 *   dev_canvas: device uint16 [canvas_h][canvas_w], caller-owned; pixels no tile covers are
 *               left untouched;  stream: cudaStream_t (NULL = legacy default stream)
 * Synchronous.  Errors: INVALID_ARG, UNSUPPORTED (n*m > 65535), CUDA.
 */
stitch_status stitch_compose_overlay(const uint16_t* dev_tiles, int32_t n, int32_t m, int32_t H,
                                     int32_t W, const int64_t* host_pos_xy, int64_t canvas_w,
                                     int64_t canvas_h, uint16_t* dev_canvas, void* stream);

/*
 * Phase 3, stream-ordered: as stitch_compose_overlay, but returns once the work is enqueued
 * on `stream` (host_pos_xy is consumed before the call returns; dev_tiles and dev_canvas
 * must stay valid until the stream reaches that point).  Errors: as above.
 */
stitch_status stitch_compose_overlay_async(const uint16_t* dev_tiles, int32_t n, int32_t m,
                                           int32_t H, int32_t W, const int64_t* host_pos_xy,
                                           int64_t canvas_w, int64_t canvas_h,
                                           uint16_t* dev_canvas, void* stream);

/* Message for the last error on ctx (valid until the next call on ctx). */
const char* stitch_last_error(stitch_ctx* ctx);

/* Release everything the context owns (NCCL communicator included).  NULL-safe. */
void stitch_destroy(stitch_ctx* ctx);

#ifdef __cplusplus
}
#endif
#endif /* STITCH_H */
