/*
 * am.h -- C ABI of the B200-native accessibility-map (AM) engine.
 *
 * One call computes the AM of one pivot: for every orientation (phi_i, gamma_j)
 * of an m x n grid, whether the tool -- N_c coaxial closed solid cylinders fixed
 * at the pivot -- collides with any of N voxels (axis-aligned cubes, centre +
 * half size).  PAPER.md L86-88 (problem statement), L56/L60 (orientation grid
 * and AM, Fig. 1-2), L311 (tool made of cylinders).  The method is AICA
 * (section 3-4, Alg. 1): per voxel, the inaccessible cone of
 * its inscribed sphere (radius h) is certainly blocked, everything outside the
 * cone of its circumscribed sphere (sqrt(3) h) is certainly clear, and the exact
 * cylinder-box test (CHECKBOX, L97) runs only in the band between the two.
 *
 * Conventions:
 *   - lengths in any consistent unit (mm in every config);
 *   - cylinder k spans axial [z_k, z_k + height_k] along the tool direction d,
 *     z_0 = 0 at the pivot, z_{k+1} = z_k + height_k (reading G3/G4);
 *   - cell (i, j): phi_i = (i + 1/2) pi / m measured from +z, gamma_j =
 *     (j + 1/2) 2 pi / n measured from +x toward +y,
 *     d = (sin phi cos gamma, sin phi sin gamma, cos phi)  (reading G1);
 *   - AM layout: W = ceil(n / 32) uint32 words per row, row-major in i; cell
 *     (i, j) is bit (j & 31) of word i * W + (j >> 5); LSB-first; padding bits
 *     are 0; 1 = collision ("black", L60)  (reading G2).
 *
 * Exactness: every cell whose oracle state is robust (exact-test margin above
 * 1e-5 rad) equals the exact definition; cells inside the 1e-5 rad
 * band may take either value.
 *
 * Ownership: the library copies whatever it is given; caller buffers are never
 * retained.  Errors: every int-returning call returns AM_OK (0) or a negative
 * AM_E* code, and am_last_error() describes the last failure on that context.
 * Threading and streams: calls on one context are not thread-safe; use one
 * context per device (per rank).  Asynchronous calls share the context's
 * scratch (per-map slots, staged pivots), so a compute call issued on another
 * stream than the previous compute call first waits (on the device) for that
 * call to finish; calls on one stream are ordered by the stream.  No call falls
 * back to the CPU: a missing or failing GPU is reported as AM_ECUDA.
 * Allocation failures (AM_ENOMEM) leave the context usable as it was: e.g. a
 * batch whose AM_OPT_BATCH slots do not fit can be retried with fewer.
 */
#ifndef AM_H_
#define AM_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct am_ctx am_ctx; /* opaque; owns all device memory of one context */

/* One bounding cylinder of the tool, ordered from the pivot outward. */
typedef struct {
    float radius; /* > 0, finite */
    float height; /* > 0, finite */
} am_cylinder;

/* Per-call counters of the AICA path (filled by am_compute when stats != NULL). */
typedef struct {
    int64_t voxels_streamed;   /* voxels read by the streaming kernel                          */
    int64_t voxels_culled;     /* beyond the tool's reach rho_max (step a2)                      */
    int64_t voxels_skipped;    /* cheap outer cone lies entirely in already-full rows (a5)      */
    int64_t voxels_live;       /* voxels whose exact cones were computed and rasterised (a4-a5) */
    int64_t rows_rasterised;   /* (voxel, phi-row) pairs rasterised                             */
    int64_t band_pairs;        /* (voxel, cell) pairs queued in the ambiguous band (a6)         */
    int64_t exact_tests;       /* exact cylinder-box tests actually run (CHECKBOX, L97)         */
    int64_t exact_hits;        /* of which collided                                             */
    int64_t queue_overflow;    /* band pairs resolved inline because the queue was full         */
    int64_t early_exit;        /* 1 if the AM filled up before the full stream, which then read
                                  no voxel (a7: "stop when popcount(AM) = m n")               */
    int64_t bricks_kept;       /* 256-voxel bricks whose voxels were read (AM_OPT_BRICKS)       */
    int64_t level_voxels;      /* voxels of the clear-map levels (read once more per map)       */
    int64_t rows_skipped_full; /* (live voxel, phi-row) pairs of the full stream skipped because
                                  the row was already full (a5: "rows already full are skipped") */
} am_stats;

enum {
    AM_OK = 0,
    AM_EINVAL = -1, /* invalid argument (see each call)                       */
    AM_ENOMEM = -2, /* device or host allocation failed                       */
    AM_ECUDA = -3,  /* CUDA runtime error (no device, launch failure, ...)    */
    AM_ESTATE = -4  /* call out of order (e.g. compute before upload)         */
};

/* Tunables (am_set_option).  Defaults are chosen at am_create. */
enum {
    AM_OPT_GRID_CTAS = 1,        /* persistent CTAs of the streaming kernel (0 = SMs x occupancy) */
    AM_OPT_REFRESH_TILES = 2,    /* tiles between shared-AM <-> global-AM merges (>= 1)          */
    AM_OPT_MORTON_SORT = 3,      /* 1 = Morton-sort voxels at upload (default), 0 = keep order   */
    AM_OPT_BASELINE_REJECT = 4,  /* 1 = baseline uses an exact-safe bounding-sphere reject        */
    AM_OPT_BAND_QUEUE = 5,       /* capacity of the deferred band queue, in (voxel, cell) pairs  */
    AM_OPT_KERNEL_TIMING = 6,    /* 1 = bracket every full-stream kernel launch with CUDA events;
                                    2 = also one event after every kernel launch (per-kernel
                                    device times, am_kernel_stats)                              */
    AM_OPT_PHASES = 7,           /* 1 = coarse levels + clear-direction map before the full
                                    stream (default); 0 = one plain stream.  Same map either way */
    AM_OPT_DIAG = 8,             /* diagnostics, 0 in production: bit 0 = stop after the coarse
                                    levels (partial map); bit 1 = seed the map and the clear-
                                    direction map with the previous map of this context instead
                                    of the coarse levels (a lower-bound probe of the filter; the
                                    result is exact only when that map had the same pivot); bit 2
                                    = per-phase times of the single-pivot kernel on stderr; bit 3
                                    = batches as one cooperative launch of CTA groups; bit 4 =
                                    am_compute with the previous single-pivot kernel (one grid
                                    barrier per phase) instead of am_latency_kernel; bit 5 =
                                    am_compute through the batched phase launches (P = 1); 0..63 */
    AM_OPT_CMAP_T = 9,           /* clear-direction map resolution: texels per cube-face side
                                    (4..256, default 96; 80 when m·n >= 128·128)                 */
    AM_OPT_BRICKS = 10,          /* 1 = skip whole 256-voxel bricks whose bounding sphere reaches
                                    no clear cell (default); 0 = read every voxel.  Same map     */
    AM_OPT_FUSED = 11,           /* 1 = the whole map in one persistent cooperative launch when
                                    phases >= 1 and bricks = 1 (default); 0 = one launch per
                                    stage.  Same map                                            */
    AM_OPT_BATCH = 12,           /* am_compute_batch: pivots computed together, phase by phase,
                                    one launch per phase (1..64, default 32; each needs its own
                                    per-map buffers, ~4 N + 100 MB of device memory).  Same maps */
    AM_OPT_BAND_SUBDIV = 13,     /* band pairs: levels of virtual 2x2x2 sub-cubes decided by
                                    CHECKICA before CHECKBOX (§4.3; 0..3,
                                    default 0 = CHECKBOX directly).  Same map outside the band  */
    AM_OPT_CMAP_T1 = 14,         /* resolution of the clear-direction map built after level 0,
                                    which only filters level 1 (4..AM_OPT_CMAP_T, default 16).
                                    Same map                                                    */
    AM_OPT_CMAP_ROWSCAN = 15,    /* clear-direction map: with more clear cells than this -- and
                                    always with more than fit in shared memory (2048) -- each
                                    texel finds its nearest clear cell row by row (nearest clear
                                    gamma per phi-row, rows outward from the texel's phi, early
                                    stop); otherwise the block / all-pairs search (0..2^21,
                                    default 1024).  Same map                                    */
    AM_OPT_CMAP_BRUTE = 16,      /* clear-direction map: with at most this many clear cells every
                                    texel tries every one; above, texel blocks first bound   
                                    the candidates from the block centre (0..2^21, default
                                    0).  Same map                                               */
    AM_OPT_CMAP_BLOCK = 17,      /* clear-direction map: side of the texel blocks (one warp each)
                                    whose centre bounds the candidate cells on that path: 4 or 8
                                    (default 8; a map resolution that is not a multiple falls
                                    back to 4, then to every texel x every cell).  Same map      */
    AM_OPT_MAP_CTAS = 18,        /* batched path: CTAs per pivot of the (final) clear-direction
                                    map launch, 0..4096 (0 = one per 1024 texels; default 48).
                                    Same map                                                    */
    AM_OPT_SUBBRICKS = 19,       /* fused and batched paths, bit 0: skip each 32-voxel sub-brick
                                    of a kept brick (one warp's voxels) whose bounding sphere
                                    reaches no clear cell before its voxels are read; bit 1
                                    (batched path): test super-bricks of 8 bricks first and only
                                    the bricks of kept ones (0..3, default 3).  Same map        */
    AM_OPT_BATCH_LANES = 20,     /* am_compute_batch: chunks of AM_OPT_BATCH / lanes pivots go
                                    round-robin to this many internal streams (forked from and
                                    joined to the caller's stream), so one chunk's short phases
                                    overlap another's (1..8, default 8; 1 while
                                    AM_OPT_KERNEL_TIMING = 2).  Same maps                       */
    AM_OPT_GRAPH = 21,           /* am_compute_batch: 1 = capture the batch's launch chain as a
                                    CUDA graph and replay it while the options, the pivot count,
                                    the output buffer and the model are unchanged (default);
                                    0 = launch every kernel from the host.  Same maps           */
    AM_OPT_L1_SAMPLE = 22,       /* coarse level 1's strided sample of the model, in voxels, taken
                                    at the NEXT am_upload_voxels (0..2^31-1; 0 = library default:
                                    every 384th voxel, at least 24,576).  Approximate: every
                                    floor(N / sample)-th voxel is taken, so the realised sample is
                                    between sample and 2 sample - 1 voxels.  Only the culling
                                    changes (scene-dependent best: profiles/r2x_level_sizes.txt).
                                    Same maps                                                   */
    AM_OPT_REUSE = 23,           /* am_compute_batch, AM reuse between neighbouring pivots
                                    ("reuse the AM values
                                    among nearby pivots"): 1 = every map slot remembers the voxels
                                    whose inner cone set new cells of its map, and the slot's next
                                    map rasterises their inner cones -- recomputed at the new pivot,
                                    so exactly -- before level 0, which tightens every clear-
                                    direction map after it.  Pays when slot s of consecutive calls
                                    gets consecutive pivots of a toolpath (e.g. call t computes
                                    pivots s L + t of 64 path segments of L pivots).  0 = off
                                    (default).  Same maps                                         */
    AM_OPT_STAGE_FUSION = 24,    /* am_compute_batch: stages run as ONE launch each whose filter
                                    survivors, cones and rows stay in shared memory (stage.cuh),
                                    by bit: 1 = level 0, 2 = level 1, 4 = the kept voxels (7 =
                                    all); a clear bit = cone and row kernels with records and
                                    tasks in device memory.  Default 1: level 0 fused (its few
                                    large cones have many rows each, and the CTA raster beats the
                                    task round trip: C3 6.33 -> 6.17 us per map); levels 1 and the
                                    kept voxels measured slower fused (their many one-thread cones
                                    leave a CTA-local drain idle: 7.3 / 9.7 us).  Same maps       */
    AM_OPT_STREAM_TMA = 25,      /* full-stream filter (AM_OPT_BRICKS = 0): north_star "voxel loads
                                    staged via TMA".  1..3 = filter_tma(_ws)_kernel: persistent CTAs
                                    whose 16 KB voxel tiles arrive in shared memory by 1-D bulk
                                    copies (cp.async.bulk completing on an mbarrier, L2 evict-first)
                                    -- 1: a producer warp refills a 2-stage ring as soon as the 8
                                    consumer warps release a stage (empty mbarriers); 2: 2 stages,
                                    thread 0 refills after a CTA barrier; 3: as 1 with 4 stages.
                                    0 = filter_kernel, 4 LDG.128 per thread (default: the filter is
                                    issue-bound, ~85 instructions per voxel, so the TMA rings measure
                                    0.56-0.61 of HBM on C3 against 0.65).  Same maps              */
    AM_OPT_PDL = 26,             /* am_compute_batch: 1 = each phase kernel of a lane is a
                                    programmatic dependent launch (griddepcontrol): its CTAs are
                                    scheduled under the previous phase's tail and copy their
                                    parameters there, then wait for the previous phase's writes
                                    (default); 0 = plain stream order.  Same maps                 */
    AM_OPT_CMAP_FAR = 27,        /* final clear-direction map, 8x8 texel blocks: a block whose
                                    centre is farther than this many degrees from every clear cell
                                    skips the per-texel nearest-clear search and stores for each
                                    texel the lower bound theta_C - angle(texel, centre) (triangle
                                    inequality; exact-safe, only less tight).  0 = never; default
                                    100 (below ~80 the looser map lets many more voxels through)
                                    Same maps                                                     */
    AM_OPT_L1_SUBS = 28,         /* am_compute_batch, coarse level 1: 1 = its voxels are kept in
                                    model (Morton) order and every 32 consecutive ones have a
                                    bounding sphere (upload); the level-1 cone launch skips a group
                                    whose sphere cannot reach a clear cell of the map after level 0;
                                    0 = every level-1 voxel filtered (default: the map after level 0
                                    is loose, few groups drop, and the sphere test costs more than it
                                    saves -- l1_cones 0.85 -> 0.90 us per map on C3).  Same maps   */
    AM_OPT_LIVE_CAP = 29,        /* am_compute_batch: live-voxel list entries per map slot, taken
                                    at the NEXT am_upload_voxels (0 = max(2^20, N / 8), at most N;
                                    default).  When a map's filter finds more live voxels, its
                                    live-cone phase streams the kept sub-bricks through the filter
                                    again and emits every live voxel's cones -- exact, only slower.
                                    Memory per slot ~4 B x this + ~100 MB (C3, 64 slots: 7.3 GB,
                                    was 13 GB).  Same maps                                        */
    AM_OPT_L1_SPARSE = 30        /* am_compute_batch: when the map after level 0 of a pivot leaves at
                                    most this many cells clear, that pivot's level 1 takes every
                                    2nd voxel (a nearly full map gains little from the rest; the
                                    coarse levels only decide what is culled).  0 = off (default:
                                    the clear count does not separate the scenes -- C5 gains 10 %
                                    only with 2^20 (always), C3 then loses 5 %; r5_sweeps.txt).
                                    Same maps                                                     */
};

/* Kernels of the library, for am_kernel_stats. */
enum {
    AM_K_L0_CONES = 0,  /* level-0 (largest voxels) inner cones, a3-a4                        */
    AM_K_L0_ROWS,       /* their phi-rows, a5                                                  */
    AM_K_CLEAR_MAP,     /* clear-direction map of the partial AM                 */
    AM_K_L1_CONES,      /* level-1 filter + inner cones                                        */
    AM_K_L1_ROWS,       /* their rows                                                          */
    AM_K_BRICKS,        /* brick bounding-sphere test, a1-a2 (8(f) NEXT 1; batched path: the
                           super-brick launch and the brick launch)                            */
    AM_K_VOXELS,        /* kept bricks' voxels through the filter -> live list, a1-a3          */
    AM_K_LIVE_CONES,    /* live voxels' inner + outer cones, a3-a4                             */
    AM_K_LIVE_ROWS,     /* their rows + band queue, a5-a7                                      */
    AM_K_BAND,          /* exact CHECKBOX of queued band pairs still clear, a6                 */
    AM_K_FUSED,         /* am_pipeline_kernel: every step of a map in one cooperative launch   */
    AM_K_FILTER,        /* full-stream filter of every voxel (AM_OPT_BRICKS = 0)               */
    AM_K_BASELINE,      /* all-pairs CHECKBOX baseline, a9                                     */
    AM_K_LAYOUT,        /* am_unpack_cells / am_pack_cells                                     */
    AM_K_ICA_MEMO,      /* am_compute_octree: parallel ICA calculation of the top S levels     */
    AM_K_OCTREE,        /* am_compute_octree: one thread per orientation, Alg. 2               */
    AM_K_INIT,          /* batched path: zero a chunk's maps and per-map counters              */
    AM_K_LEVEL0,        /* batched, AM_OPT_STAGE_FUSION: level 0 (+ reuse witnesses), cones + rows  */
    AM_K_LEVEL1,        /* batched, AM_OPT_STAGE_FUSION: level-1 filter, cones + rows             */
    AM_K_STREAM,        /* batched, AM_OPT_STAGE_FUSION: kept voxels' filter, cones, rows, band queue */
    AM_K_COUNT
};

/*
 * Create a context on CUDA device `device` for the tool `tool[0..n_cyl)` and an
 * m x n orientation grid.  AM_EINVAL unless 1 <= n_cyl <= 8, every radius and
 * height is finite and > 0, 1 <= m <= 1024, 1 <= n <= 1024 and out != NULL.
 * AM_ECUDA if the device cannot be used.  On success *out owns the context.
 */
int am_create(const am_cylinder* tool, int n_cyl, int m, int n, int device, am_ctx** out);

/*
 * Upload the voxel model: N voxels with centres centers_xyz[3*N] (x, y, z
 * interleaved) and half sizes half_sizes[N], both float32, on the host
 * (src_is_device = 0) or on `device` (1).  Replaces any previous model.  The
 * library may reorder voxels (Morton sort); the AM is order-independent.
 * AM_EINVAL if N < 0, a pointer is NULL while N > 0, or any value is non-finite
 * or a half size is <= 0.  N = 0 is legal (every AM is then all-zero).  A failed
 * upload leaves no model: compute calls return AM_ESTATE until an upload succeeds.
 * Synchronous: returns after the model is resident (upload time is excluded
 * from AM timings).
 */
int am_upload_voxels(am_ctx* ctx, const float* centers_xyz, const float* half_sizes, int64_t N,
                     int src_is_device);

/*
 * AICA accessibility map of one pivot (host array pivot[3], finite).
 * am_out receives am_words_per_map(ctx) uint32 words in the layout above, in
 * host memory (dst_is_device = 0; the call then synchronises the stream) or in
 * device memory (1; the call is asynchronous on `cuda_stream`).  cuda_stream is
 * a cudaStream_t (NULL = legacy default stream).  stats, if non-NULL, is filled
 * (this synchronises the stream).  AM_ESTATE before am_upload_voxels.
 */
int am_compute(am_ctx* ctx, const float pivot[3], uint32_t* am_out, int dst_is_device,
               void* cuda_stream, am_stats* stats);

/*
 * AMs of P pivots (host array pivots[3*P]); am_out receives P consecutive maps
 * of am_words_per_map(ctx) words each (host or device as above).  Same maps as
 * P calls of am_compute (the toolpath batch of SURVEY.md 8(e)(2)); up to
 * AM_OPT_BATCH pivots run together, one launch per phase (8(f) NEXT 2).
 */
int am_compute_batch(am_ctx* ctx, const float* pivots, int64_t P, uint32_t* am_out,
                     int dst_is_device, void* cuda_stream);

/*
 * Baseline AM of one pivot: the exact cylinder-box test (CHECKBOX, PAPER.md
 * L97, Fig. 4 L82) for every (voxel, orientation) pair, without cones -- the
 * non-pruned analogue of the paper's PBox (L269).  Per orientation the scan
 * stops at the first collision (Alg. 2).  Same output contract as
 * am_compute.
 */
int am_compute_baseline(am_ctx* ctx, const float pivot[3], uint32_t* am_out, int dst_is_device,
                        void* cuda_stream);

/* Set a tunable (AM_OPT_*).  AM_EINVAL for an unknown key or an out-of-range value. */
int am_set_option(am_ctx* ctx, int key, int64_t value);

/*
 * Device time of the dominant kernel summed over its launches since the
 * previous call: the fused pipeline kernel (am_pipeline_kernel, every step of
 * the map in one launch) when AM_OPT_FUSED applies, otherwise the full-stream
 * launch of steps a1-a3 (brick_test + brick_voxels, or filter_kernel when
 * AM_OPT_BRICKS = 0).  Measured with CUDA events recorded on the launching
 * stream while AM_OPT_KERNEL_TIMING is 1.  Waits for
 * the recorded events, then resets the accumulator.  *total_ms and *launches
 * must be non-NULL.
 */
int am_kernel_time(am_ctx* ctx, double* total_ms, int64_t* launches);

/*
 * Per-kernel accounting since the previous call, indexed by AM_K_*: ms[k] =
 * device time of kernel k's launches (only while AM_OPT_KERNEL_TIMING = 2,
 * else 0: consecutive CUDA events on the launching stream, one after every
 * launch, so a launch's interval also holds the gap before it), launches[k] =
 * how many times kernel k was launched by any call (counted always).  Both
 * arrays hold AM_K_COUNT entries, caller-owned.  Waits for the recorded
 * events, then resets.  AM_EINVAL for NULL outputs.
 */
int am_kernel_stats(am_ctx* ctx, double* ms, int64_t* launches);

/* Name of kernel k (static string), NULL if k is not an AM_K_* value. */
const char* am_kernel_name(int k);

/*
 * The paper's own GPU schemes (§4),
 * for comparison with am_compute: one thread per orientation traverses the
 * octree with Alg. 2 CHECKOCTREE (L198-221) using the scheme's elementary test.
 * All give the same map as am_compute outside the 1e-5 rad band (each falls
 * back to the exact test); they differ in work.
 */
enum {
    AM_SCHEME_PBOX = 0,       /* CHECKBOX on every visited node (the baseline, L269)          */
    AM_SCHEME_PBOX_AABB = 1,  /* optimized PBox: rotated-box AABB reject first (L268)         */
    AM_SCHEME_PICA = 2,       /* CHECKICA computed on the fly, CHECKBOX for corner cases      */
    AM_SCHEME_MICA = 3,       /* + cones of the top S levels memoised in parallel (§4.2)      */
    AM_SCHEME_AICA = 4        /* + corner cases expanded into children (§4.3)        */
};

/*
 * Build the octree (root + interior + leaves) of the resident
 * model.  The uploaded voxels must be the leaves of an adaptive octree whose
 * root cube is [root_lo, root_lo + root_size]^3: every half size is
 * root_size / 2^(l+1) for a level 0 <= l <= 20 and every centre the centre of
 * a level-l cell; the cells must be disjoint.  AM_EINVAL otherwise (and for a
 * non-finite or non-positive root), AM_ESTATE before am_upload_voxels.
 * Interior nodes are the cells that contain leaves; children are stored
 * contiguously, nodes in level (BFS) order.  *n_nodes (nullable) receives the
 * node count.  Synchronous; a new upload discards the octree.
 */
int am_build_octree(am_ctx* ctx, const float root_lo[3], float root_size, int64_t* n_nodes);

/*
 * AM of one pivot with scheme AM_SCHEME_* over the octree (same output
 * contract as am_compute).  S = levels whose cones are memoised by the
 * parallel ICA calculation (MICA / AICA; 0..64, levels 0..S-1), vdepth =
 * AICA's virtual expansion depth of band leaves before CHECKBOX (0..3).
 * stats (nullable, 4 entries): nodes popped, CHECKBOX calls, on-the-fly ICA
 * evaluations, max nodes popped by one thread (the critical thread of Fig. 13
 * L323); filling it synchronises the stream.  AM_EINVAL for a bad scheme, S or
 * vdepth; AM_ESTATE before am_build_octree.
 */
int am_compute_octree(am_ctx* ctx, const float pivot[3], int scheme, int S, int vdepth, uint32_t* am_out,
                      int dst_is_device, void* cuda_stream, int64_t* stats);

/*
 * Layout conversion on the device, for the voxel-sharded multi-GPU combine
 * (SURVEY.md 8(e)(1)): an all_reduce(MAX) over one byte per cell is the OR of
 * the ranks' maps, which MAX over packed words is not.
 *   am_unpack_cells: words (m * ceil(n/32) uint32, layout above) -> cells
 *                    (m * n uint8, row-major, 0/1);
 *   am_pack_cells:   cells (nonzero = collision) -> words.
 * Both pointers are device memory of ctx's device; asynchronous on
 * cuda_stream.  AM_EINVAL for NULL pointers.
 */
int am_unpack_cells(am_ctx* ctx, const uint32_t* words, uint8_t* cells, void* cuda_stream);
int am_pack_cells(am_ctx* ctx, const uint8_t* cells, uint32_t* words, void* cuda_stream);

/* m * ceil(n / 32): words per AM.  -1 if ctx is NULL. */
int am_words_per_map(const am_ctx* ctx);

/* Number of voxels currently resident (-1 if ctx is NULL). */
int64_t am_num_voxels(const am_ctx* ctx);

/* Human-readable description of the last error on ctx (never NULL). */
const char* am_last_error(const am_ctx* ctx);

/* Free the context and all its device memory.  NULL is a no-op. */
void am_destroy(am_ctx* ctx);

#ifdef __cplusplus
}
#endif

#endif /* AM_H_ */
