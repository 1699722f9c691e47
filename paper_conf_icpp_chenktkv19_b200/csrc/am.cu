// am.cu -- host side of the C ABI declared in include/am.h (L1 of SURVEY.md 1).
//
// Owns the device state of one context: the resident voxel list (float4,
// Morton-sorted at upload), the orientation tables, the band queue, a scratch
// AM and the per-call counters.  Every entry point validates its arguments,
// launches sm_100a kernels on the caller's stream and reports CUDA failures as
// AM_ECUDA.  There is no CPU fallback.
#include <cuda_runtime.h>

#include <cub/device/device_radix_sort.cuh>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <string>
#include <vector>

#include "../../include/am.h"
#include "kernels.cuh"
#include "stream.cuh"
#include "fused.cuh"
#include "batch.cuh"
#include "latency.cuh"
#include "stage.cuh"
#include "octree.cuh"

#include <algorithm>
#include <cstdint>

using namespace am;

// coarse-level sizes (upload): level 0 = the N / AM_L0_DIV largest voxels,
// level 1 = the next up to N / AM_L1_DIV plus every AM_L1_STRIDE-th voxel (a sample of at
// least AM_L1_MIN_SAMPLE voxels: small models, tools/ab.sh on C2)
#ifndef AM_ROWS_CTAS
#define AM_ROWS_CTAS 64
#endif
#ifndef AM_VOXEL_CTAS
#define AM_VOXEL_CTAS 32  // CTAs per pivot of bk_voxels (swept on B200 with PDL: profiles/r5_sweeps.txt)
#endif
#ifndef AM_CONE_CTAS
#define AM_CONE_CTAS 64
#endif
#ifndef AM_BATCH_LANES
#define AM_BATCH_LANES 8
#endif
constexpr int kMaxLanes = 8;
#ifndef AM_L1_STEPS
#define AM_L1_STEPS 8  // level-1 cone steps (256 voxels each) per CTA of the batched path
#endif
#ifndef AM_BRICKS_CTAS
#define AM_BRICKS_CTAS 16  // per pivot, brick launch after the super-brick test (entries = 8 x kept supers)
#endif
#ifndef AM_BRICK_STEPS
#define AM_BRICK_STEPS 4  // brick-test steps (256 bricks each) per CTA of the batched path
#endif
#ifndef AM_MAP_CTAS
#define AM_MAP_CTAS 48
#endif
#ifndef AM_CMAP_BLOCK
#define AM_CMAP_BLOCK 8
#endif
#ifndef AM_CMAP_BRUTE
#define AM_CMAP_BRUTE 0
#endif
#ifndef AM_CMAP_ROWSCAN
#define AM_CMAP_ROWSCAN 1024
#endif
#ifndef AM_CMAP_FAR
#define AM_CMAP_FAR 100  // degrees (AM_OPT_CMAP_FAR; swept on B200: profiles/r5_sweeps.txt)
#endif
#ifndef AM_CMAP_T1
#define AM_CMAP_T1 16  // (32 before; 16 equal or faster on every config, batched and single pivot: profiles/r5_sweeps.txt)
#endif
#ifndef AM_FUSED_BRICKS
#define AM_FUSED_BRICKS 1  // batched: bk_bricks_fused instead of bk_supers + bk_bricks (r5_sweeps.txt)
#endif
#ifndef AM_FUSED_BRICKS_SUPERS
#define AM_FUSED_BRICKS_SUPERS 512  // super-bricks per CTA of bk_bricks_fused (2 per thread)
#endif
#ifndef AM_L0_PER_CTA
#define AM_L0_PER_CTA 256
#endif
#ifndef AM_L0_CTAS
#define AM_L0_CTAS 32
#endif
#ifndef AM_MAP1_WARP_TEXEL
#define AM_MAP1_WARP_TEXEL 0
#endif
#ifndef AM_MAP1_WARP_BLOCKS
#define AM_MAP1_WARP_BLOCKS 4
#endif
#ifndef AM_BAND_CTAS
#define AM_BAND_CTAS 24
#endif
#ifndef AM_BAND_THREADS
#define AM_BAND_THREADS 256
#endif
#ifndef AM_L0_DIV
#define AM_L0_DIV 16384
#endif
#ifndef AM_L1_DIV
#define AM_L1_DIV 4096
#endif
#ifndef AM_L1_STRIDE
#define AM_L1_STRIDE 384
#endif
#ifndef AM_L1_MIN_SAMPLE
#define AM_L1_MIN_SAMPLE 24576
#endif

// AM_OPT_STREAM_TMA ring shapes of filter_tma_kernel: (voxels per thread per tile, stages)
// AM_OPT_STREAM_TMA values: ring shapes of the TMA-staged full-stream filter (stream.cuh), as
// (voxels per thread per tile, stages); measured on B200 (C3, profiles/r5_tma_sweep.txt) all below
// the LDG filter_kernel, which is the default (0)
constexpr int kTmaShapes = 3;
inline const void* tma_kernel(int k) {
    switch (k) {
        case 1: return (const void*)filter_tma_ws_kernel<4, 2>;  // warp-specialised producer, 32 KB ring
        case 2: return (const void*)filter_tma_kernel<4, 2>;     // CTA barrier per tile, 32 KB ring
        default: return (const void*)filter_tma_ws_kernel<4, 4>; // warp-specialised producer, 64 KB ring
    }
}
inline int tma_stages(int k) { return k == 3 ? 4 : 2; }
inline size_t tma_smem(int k) { return (size_t)tma_stages(k) * 4 * kThreads * sizeof(float4); }
inline int tma_threads(int k) { return k == 2 ? kThreads : kThreads + 32; }
inline long long tma_tile_vox(int) { return 4ll * kThreads; }

struct am_ctx {
    int device = 0;
    int sms = 0;
    ToolDev tool{};
    GridDev grid{};
    int MW = 0;
    // resident model
    float4* d_vox = nullptr;
    long long N = 0;
    long long vox_cap = 0;
    long long live_cap = 0;                // live list entries per map slot (d_live holds slots x live_cap)
    long long live_cap_opt = 0;            // AM_OPT_LIVE_CAP (0 = max(2^20, N / 8), at most N)
    bool uploaded = false;
    // per-call state
    float* d_tab = nullptr;                // cos phi, sin phi, cos gamma, sin gamma
    uint32_t* d_am = nullptr;              // scratch AM(s) for host destinations
    long long am_cap_maps = 0;
    unsigned long long* d_ctr = nullptr;   // [0] queue count, [1..] stats
    unsigned long long* d_queue = nullptr;
    long long qcap = 0;
    // options
    int grid_ctas = 0;
    int refresh_tiles = 8;
    int morton = 1;
    int baseline_reject = 0;
    size_t smem = 0, smem_coarse = 0, smem_cmap = 0;
    int occ = 0;
    // coarse levels (largest voxels + a strided sample) and the clear-direction map
    float4* d_coarse = nullptr;
    float4* d_l1subs = nullptr;            // bounding spheres of every 32 consecutive level-1 voxels
    int l1_subs = 0;                       // AM_OPT_L1_SUBS: level-1 groups of 32 culled by their sphere
    int l1_sparse = 0;                     // AM_OPT_L1_SPARSE: clear cells after level 0 up to which level 1 is halved
    unsigned int* d_live = nullptr;        // live-voxel lists of the batched map slots (slots x live_cap)
    unsigned int* d_live_full = nullptr;   // live-voxel list of the single-pivot paths (capacity N)
    ConeRec* d_recs = nullptr;             // cone records (kRecCap) and row tasks (kTaskCap)
    unsigned long long* d_tasks = nullptr;
    long long n_l0 = 0, n_l1 = 0;          // level 0 = [0, n_l0), level 1 = [n_l0, n_l1)
    float4* d_texels = nullptr;            // cube-map texel centres (xyz) + angular radius (w)
    float4* d_cmap = nullptr;              // per slot: per texel (cos, sin of the nearest-clear angle, U_t |U_t|, 0)
    float4* d_cmap_ones = nullptr;         // the all-clear map (no voxel can be dropped): (1, 0, 1, 0)
    uint32_t* d_prev = nullptr;            // diagnostics: copy of the last map
    unsigned long long* d_ts = nullptr;    // diagnostics: fused-phase timestamps
    int diag = 0;
    int diag_ts = 0;
    int cmapT = 96;
    long long l1_sample = 0;               // AM_OPT_L1_SAMPLE (0 = N / AM_L1_STRIDE, >= AM_L1_MIN_SAMPLE)
    int cmapT1 = AM_CMAP_T1;               // map after level 0 (AM_OPT_CMAP_T1, <= cmapT)
    float4* d_texels1 = nullptr;
    int phases = 2;
    float4* d_bricks = nullptr;            // bounding spheres of 256-voxel bricks of d_vox
    unsigned int* d_brick_list = nullptr;  // kept bricks (stream path) / sub-bricks (fused path) per map (capacity 8 nbricks)
    unsigned int nbricks = 0;
    int bricks_on = 1;
    float4* d_subs = nullptr;              // bounding spheres of 32-voxel sub-bricks (warps of a brick)
    float4* d_supers = nullptr;            // bounding spheres of 2048-voxel super-bricks (8 bricks)
    int subs_on = 3;                       // AM_OPT_SUBBRICKS: bit 0 sub-bricks, bit 1 super-bricks
    int fused = 1;                         // one cooperative launch per map (fused.cuh)
    int batch = 32;                        // pivots per batched launch (AM_OPT_BATCH)
    int band_vdepth = 0;                   // AM_OPT_BAND_SUBDIV
    int bk_rows_ctas = AM_ROWS_CTAS, bk_voxel_ctas = AM_VOXEL_CTAS, bk_cone_ctas = AM_CONE_CTAS;  // per pivot, batched phases
    int lanes = AM_BATCH_LANES;            // streams of the batched path (AM_OPT_BATCH_LANES)
    int use_graph = 1;                     // AM_OPT_GRAPH: replay the batched launch chain as a CUDA graph
    unsigned long long gen = 1;            // bumped by every option / upload / reallocation (graph key)
    cudaStream_t cap_s = nullptr;          // capture stream
    cudaGraphExec_t g_exec = nullptr;      // the captured chain and its key
    unsigned long long g_gen = 0;
    int64_t g_P = 0;
    const void* g_piv = nullptr;
    long long g_launches[AM_K_COUNT] = {};  // kernel launches per replay (am_kernel_stats)
    cudaStream_t lane_s[kMaxLanes] = {};
    cudaEvent_t lane_ev[kMaxLanes + 1] = {};
    int bk_map_ctas = AM_MAP_CTAS;         // per pivot, batched clear map (AM_OPT_MAP_CTAS; 0 = texels / 1024)
    int slots = 1;                         // per-map buffer slots allocated (d_ctr ... d_brick_list)
    float4* d_piv = nullptr;               // batched launch: pivots (xyz, may_cull)
    long long piv_cap = 0;
    float4* h_piv = nullptr;               // pinned staging of the batch's pivots (xyz, may_cull)
    long long h_piv_cap = 0;
    cudaEvent_t piv_ev = nullptr;          // the last pivot upload (the staging is reused after it)
    cudaEvent_t done_ev = nullptr;         // end of the last compute call (its stream: last_s)
    cudaStream_t last_s = nullptr;
    bool has_last = false;
    unsigned long long* d_bctl = nullptr;  // batched launch: group barriers, pivot queue
    int fused_grid = 0;
    int lat_grid = 0;                      // am_latency_kernel: co-resident CTAs (cooperative launch)
    // AM_OPT_REUSE (8(f) NEXT 2): per slot, two per-cell witness arrays and a dedupe set
    int reuse = 0;
    int stage_fusion = 1;                  // AM_OPT_STAGE_FUSION: stages (bit 0 level 0, 1 level 1, 2 kept voxels) as one kernel each (stage.cuh)
    int stream_tma = 0;                    // AM_OPT_STREAM_TMA: full-stream filter with TMA-staged tiles
    int pdl = 1;                           // AM_OPT_PDL: batched phases as programmatic dependent launches
    int occ_tma[8] = {};                   // filter_tma_kernel: CTAs per SM, per ring shape
    unsigned int* d_wit = nullptr;         // slots x 2 x m n voxel ids
    unsigned int* d_hash = nullptr;        // slots x hash_words
    unsigned int hash_words = 0;
    int contrib_slots = 0;
    unsigned int reuse_parity = 0;         // the list this call writes (the other is read)
    size_t smem_fused = 0;
    float bbox[6] = {0, 0, 0, 0, 0, 0};    // centre bounding box of the resident model
    // kernel timing (AM_OPT_KERNEL_TIMING)
    int timing = 0;
    std::vector<cudaEvent_t> ev_start, ev_stop;
    size_t ev_used = 0;
    // per-kernel accounting (am_kernel_stats): launches always, device time
    // while AM_OPT_KERNEL_TIMING = 2 (an event after every launch, chained)
    long long k_launches[AM_K_COUNT] = {};
    std::vector<cudaEvent_t> kev;          // event pool
    size_t kev_used = 0;
    long long kev_prev = -1;               // chain: event recorded before the next launch
    std::vector<std::pair<int, size_t>> kmarks;  // (kernel, index of its end event)
    std::vector<size_t> kmark_begin;
    // octree of the resident model (am_build_octree; paper-faithful schemes)
    float4* d_onode = nullptr;             // node cubes, BFS order
    int2* d_olink = nullptr;               // (first child, child count)
    float4* d_omemo = nullptr;             // memoised cones of the top levels
    unsigned long long* d_ostats = nullptr;
    long long o_n = 0;
    bool o_built = false;
    std::vector<long long> o_level_end;    // nodes of levels <= L: [0, o_level_end[L])
    std::string err;
};

namespace {

// d_ctr layout (64-bit words, zeroed once per map): [0] band-queue count,
// [1, 1 + ST_COUNT) am_stats of the full stream, then the per-stage counters,
// then scratch stats for the clear-map levels.
constexpr int kCtrTiles = 1 + ST_COUNT;      // live count: full stream (+0), level 1 (+4)
constexpr int kCtrRT = kCtrTiles + 5;        // stage s: record count at +2s, task count at +2s+1
constexpr int kCtrBricks = kCtrRT + 6;       // bricks kept by brick_test_kernel
constexpr int kCtrSupers = kCtrBricks + 1;   // super-bricks kept (batched path)
constexpr int kCtrClear1 = kCtrSupers + 1;   // clear cells after level 0 (batched path, AM_OPT_L1_SPARSE)
constexpr int kCtrWords = kCtrClear1 + 1;
constexpr int kCtrAll = kCtrWords + ST_COUNT;  // + scratch stats of the clear-map levels
constexpr int kCtrStride = kCtrAll;          // 64-bit words per slot
constexpr int kMaxBatch = 64;                // pivots per layered batch launch (slots)
constexpr int kBctlWords = 2 * kMaxSlots + 1 + kMaxSlots / 2;  // bars, then queue head + per-group pivot (u32)
constexpr unsigned int kRecCap = 1u << 20;   // cone records per stage (more: rows rasterised inline)
constexpr unsigned long long kTaskCap = 1ull << 22;  // (voxel, row) tasks per stage

int fail(am_ctx* c, int code, const char* fmt, ...) {
    if (c) {
        char buf[512];
        va_list ap;
        va_start(ap, fmt);
        vsnprintf(buf, sizeof buf, fmt, ap);
        va_end(ap);
        c->err = buf;
    }
    return code;
}

#define CK(call)                                                                              \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess) {                                                              \
            cudaGetLastError();                                                               \
            return fail(ctx, e_ == cudaErrorMemoryAllocation ? AM_ENOMEM : AM_ECUDA, "%s: %s (%s:%d)", \
                        #call, cudaGetErrorString(e_), __FILE__, __LINE__);                  \
        }                                                                                     \
    } while (0)

int kchain(am_ctx* ctx, cudaStream_t s);
int kmark(am_ctx* ctx, cudaStream_t s, int k);

// Restores the caller's current device on scope exit.
struct DeviceGuard {
    int prev = -1;
    bool ok = false;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) == cudaSuccess && cudaSetDevice(dev) == cudaSuccess) ok = true;
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

bool is_finite_f(float x) { return std::isfinite(x); }

StreamParams make_params(am_ctx* c, const float pivot[3], uint32_t* gam) {
    StreamParams p{};
    p.tool = c->tool;
    p.grid = c->grid;
    p.px = pivot[0];
    p.py = pivot[1];
    p.pz = pivot[2];
    p.vox = c->d_vox;
    p.N = c->N;
    p.gam = gam;
    p.tab = c->d_tab;
    p.qcount = c->d_ctr;
    p.stats = c->d_ctr + 1;
    p.early = c->d_ctr + 1 + ST_EARLY;
    p.queue = c->d_queue;
    p.qcap = c->qcap;
    p.refresh_tiles = c->refresh_tiles;
    p.vox_main = c->d_vox;
    p.vox_coarse = c->d_coarse;
    p.live_cap = (unsigned int)c->vox_cap;  // (d_live_full; the batched path overrides both)
    p.cmapT = c->cmapT;
    p.cmap_tex = c->d_texels;
    p.cull_dist = c->tool.rho_max * (1.f + 1e-5f) + 1e-6f;
    p.band_vdepth = c->band_vdepth;
    // the reach cull can only fire when some voxel centre lies farther than
    // cull_dist from the pivot: compare with the farthest corner of the bbox
    double far2 = 0.0;
    for (int k = 0; k < 3; ++k) {
        const double d = std::max(std::fabs((double)c->bbox[k] - pivot[k]), std::fabs((double)c->bbox[3 + k] - pivot[k]));
        far2 += d * d;
    }
    p.may_cull = std::sqrt(far2) * (1.0 + 1e-6) + 1e-6 > (double)p.cull_dist;
    return p;
}

// Cube-map texels: centre direction and an angular radius bounding every
// direction cube_texel() maps into the texel (max angle to the 4 corners of a
// convex spherical quadrilateral, plus slack for fp32 rounding at the edges).
std::vector<float> make_texels(int T) {
    std::vector<float> out((size_t)6 * T * T * 4);
    auto dir = [](int face, double u, double w, double* d) {
        const int a = face >> 1;
        const double sg = (face & 1) ? -1.0 : 1.0;
        double v[3];
        if (a == 0) { v[0] = sg; v[1] = u; v[2] = w; }
        else if (a == 1) { v[0] = u; v[1] = sg; v[2] = w; }
        else { v[0] = u; v[1] = w; v[2] = sg; }
        const double nn = std::sqrt(v[0] * v[0] + v[1] * v[1] + v[2] * v[2]);
        for (int k = 0; k < 3; ++k) d[k] = v[k] / nn;
    };
    for (int f = 0; f < 6; ++f)
        for (int iw = 0; iw < T; ++iw)
            for (int iu = 0; iu < T; ++iu) {
                const double u0 = -1.0 + 2.0 * iu / T, u1 = -1.0 + 2.0 * (iu + 1) / T;
                const double w0 = -1.0 + 2.0 * iw / T, w1 = -1.0 + 2.0 * (iw + 1) / T;
                double c[3];
                dir(f, 0.5 * (u0 + u1), 0.5 * (w0 + w1), c);
                double r = 0.0;
                const double us[2] = {u0, u1}, ws[2] = {w0, w1};
                for (double uu : us)
                    for (double ww : ws) {
                        double d[3];
                        dir(f, uu, ww, d);
                        const double dp = std::min(1.0, c[0] * d[0] + c[1] * d[1] + c[2] * d[2]);
                        r = std::max(r, std::acos(dp));
                    }
                const size_t t = ((size_t)(f * T + iw) * T + iu) * 4;
                out[t] = (float)c[0];
                out[t + 1] = (float)c[1];
                out[t + 2] = (float)c[2];
                out[t + 3] = (float)(r + 2e-5);
            }
    // the clear map's 8 x 8-texel blocks (kernels.cuh clear_map_blocks), 2 float4 each after
    // the texels: (c, cos 2rho'), (sin 2rho', 0, 0, 0) with c the normalised sum of the
    // block's (fp32) texel centres and 2rho' = 2 max angle(c, texel centre) + 1e-6 + 1e-4
    if (T % 8 == 0) {
        const int Tc = T / 8;
        const size_t ntex = (size_t)6 * T * T;
        out.resize((ntex + (size_t)2 * 6 * Tc * Tc) * 4, 0.f);
        for (int ct = 0; ct < 6 * Tc * Tc; ++ct) {
            const int f = ct / (Tc * Tc), rem = ct % (Tc * Tc), cw = rem / Tc, cu = rem % Tc;
            double sum[3] = {0, 0, 0};
            for (int a = 0; a < 8; ++a)
                for (int b = 0; b < 8; ++b) {
                    const size_t t = ((size_t)(f * T + 8 * cw + a) * T + 8 * cu + b) * 4;
                    for (int k = 0; k < 3; ++k) sum[k] += (double)out[t + k];
                }
            const double nn = std::sqrt(sum[0] * sum[0] + sum[1] * sum[1] + sum[2] * sum[2]);
            float cf[3];
            for (int k = 0; k < 3; ++k) cf[k] = (float)(sum[k] / nn);
            double rho = 0.0;
            for (int a = 0; a < 8; ++a)
                for (int b = 0; b < 8; ++b) {
                    const size_t t = ((size_t)(f * T + 8 * cw + a) * T + 8 * cu + b) * 4;
                    const double d0 = out[t], d1 = out[t + 1], d2 = out[t + 2];
                    const double dn = std::sqrt(d0 * d0 + d1 * d1 + d2 * d2);
                    const double cn = std::sqrt((double)cf[0] * cf[0] + (double)cf[1] * cf[1] + (double)cf[2] * cf[2]);
                    const double dp = (cf[0] * d0 + cf[1] * d1 + cf[2] * d2) / (dn * cn);
                    rho = std::max(rho, std::acos(std::max(-1.0, std::min(1.0, dp))));
                }
            const double a2 = 2.0 * (rho + 1e-6) + 1e-4;
            const size_t o = (ntex + 2 * (size_t)ct) * 4;
            out[o] = cf[0];
            out[o + 1] = cf[1];
            out[o + 2] = cf[2];
            out[o + 3] = (float)std::cos(a2);
            out[o + 4] = (float)std::sin(a2);
        }
    }
    return out;
}

// Words per slot of d_brick_list: kept sub-bricks (8 per brick), then kept super-bricks.
unsigned long long blist_words(const am_ctx* ctx) {
    return 8ull * ctx->nbricks + (ctx->nbricks + 7) / 8;
}

// (all-or-nothing, like ensure_slots: on failure the previous queue stays)
int ensure_queue(am_ctx* ctx, long long cap) {
    if (ctx->d_queue && ctx->qcap == cap) return AM_OK;
    unsigned long long* q = nullptr;
    CK(cudaMalloc(&q, (size_t)ctx->slots * cap * sizeof(unsigned long long)));
    if (ctx->d_queue) {
        cudaDeviceSynchronize();
        cudaFree(ctx->d_queue);
    }
    ctx->d_queue = q;
    ctx->qcap = cap;
    ++ctx->gen;
    return AM_OK;
}

// Texels of the map after level 0 (T1 texels per face, T1 <= cmapT: the map
// lives in the first 6 T1^2 floats of the slot's cmap).  All-or-nothing.
int set_texels1(am_ctx* ctx, int T1) {
    const std::vector<float> tex = make_texels(T1);
    float4* t = nullptr;
    CK(cudaMalloc(&t, tex.size() * sizeof(float)));
    const cudaError_t e = cudaMemcpy(t, tex.data(), tex.size() * sizeof(float), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
        cudaFree(t);
        CK(e);
    }
    cudaDeviceSynchronize();
    cudaFree(ctx->d_texels1);
    ctx->d_texels1 = t;
    ctx->cmapT1 = T1;
    ++ctx->gen;
    return AM_OK;
}

// Clear-direction map resolution T (AM_OPT_CMAP_T): texel table, per-slot maps and the all-clear
// map, all-or-nothing; then the level-0 map's texels at min(T1, T).
int set_cmap_T(am_ctx* ctx, int T) {
    const std::vector<float> tex = make_texels(T);
    const std::vector<float4> ones(tex.size() / 4, make_float4(1.f, 0.f, 1.f, 0.f));
    float4 *t = nullptr, *cm = nullptr, *on = nullptr;
    cudaError_t e = cudaMalloc(&t, tex.size() * sizeof(float));
    if (e == cudaSuccess) e = cudaMalloc(&cm, (size_t)ctx->slots * ones.size() * sizeof(float4));
    if (e == cudaSuccess) e = cudaMalloc(&on, ones.size() * sizeof(float4));
    if (e == cudaSuccess) e = cudaMemcpy(t, tex.data(), tex.size() * sizeof(float), cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMemcpy(on, ones.data(), ones.size() * sizeof(float4), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
        cudaGetLastError();
        cudaFree(t);
        cudaFree(cm);
        cudaFree(on);
        return fail(ctx, e == cudaErrorMemoryAllocation ? AM_ENOMEM : AM_ECUDA, "cmap_T %d: %s", T,
                    cudaGetErrorString(e));
    }
    cudaDeviceSynchronize();
    cudaFree(ctx->d_texels);
    cudaFree(ctx->d_cmap);
    cudaFree(ctx->d_cmap_ones);
    ctx->d_texels = t;
    ctx->d_cmap = cm;
    ctx->d_cmap_ones = on;
    ctx->cmapT = T;
    ++ctx->gen;
    return set_texels1(ctx, std::min(ctx->cmapT1, ctx->cmapT));
}

// Per-map buffers for K slots (slot s of each = the buffer of pivot s of a
// batched launch; the single-map paths use slot 0).
// All-or-nothing: the new buffers are allocated first and swapped in only when every
// allocation succeeded, so an AM_ENOMEM leaves the context as it was (its current slots
// stay usable, e.g. for a retry with a smaller AM_OPT_BATCH).
int ensure_slots(am_ctx* ctx, int K) {
    if (ctx->slots >= K) return AM_OK;
    const size_t ntex = (size_t)6 * ctx->cmapT * ctx->cmapT;
    unsigned long long *ctr = nullptr, *queue = nullptr, *tasks = nullptr;
    ConeRec* recs = nullptr;
    float4* cmap = nullptr;
    unsigned int *live = nullptr, *blist = nullptr;
    cudaError_t e = cudaSuccess;
    auto al = [&](void** p, size_t bytes) {
        if (e == cudaSuccess && bytes > 0) e = cudaMalloc(p, bytes);
    };
    al((void**)&ctr, (size_t)K * kCtrStride * sizeof(unsigned long long));
    al((void**)&queue, (size_t)K * ctx->qcap * sizeof(unsigned long long));
    al((void**)&recs, (size_t)K * kRecCap * sizeof(ConeRec));
    al((void**)&tasks, (size_t)K * kTaskCap * sizeof(unsigned long long));
    al((void**)&cmap, (size_t)K * ntex * sizeof(float4));
    if (ctx->live_cap > 0) al((void**)&live, (size_t)K * ctx->live_cap * sizeof(unsigned int));
    if (ctx->nbricks > 0) al((void**)&blist, (size_t)K * blist_words(ctx) * sizeof(unsigned int));
    if (e == cudaSuccess) e = cudaMemset(ctr, 0, (size_t)K * kCtrStride * sizeof(unsigned long long));
    if (e != cudaSuccess) {
        cudaGetLastError();
        cudaFree(ctr); cudaFree(queue); cudaFree(recs); cudaFree(tasks); cudaFree(cmap); cudaFree(live); cudaFree(blist);
        return fail(ctx, e == cudaErrorMemoryAllocation ? AM_ENOMEM : AM_ECUDA,
                    "%d map slots need ~%.1f GB of device memory: %s (the context keeps its %d slots)", K,
                    (double)K * (kCtrStride * 8.0 + ctx->qcap * 8.0 + kRecCap * sizeof(ConeRec) + kTaskCap * 8.0 +
                                 ntex * 16.0 + ctx->live_cap * 4.0 + blist_words(ctx) * 4.0) / 1e9,
                    cudaGetErrorString(e), ctx->slots);
    }
    CK(cudaDeviceSynchronize());  // no launch may still use the old buffers
    cudaFree(ctx->d_ctr); cudaFree(ctx->d_queue); cudaFree(ctx->d_recs); cudaFree(ctx->d_tasks);
    cudaFree(ctx->d_cmap); cudaFree(ctx->d_live); cudaFree(ctx->d_brick_list);
    ctx->d_ctr = ctr;
    ctx->d_queue = queue;
    ctx->d_recs = recs;
    ctx->d_tasks = tasks;
    ctx->d_cmap = cmap;
    ctx->d_live = live;
    ctx->d_brick_list = blist;
    ctx->slots = K;
    ++ctx->gen;
    return AM_OK;
}

int configure_launch(am_ctx* ctx) {
    const int m = ctx->grid.m;
    ctx->smem = live_smem_bytes(m, ctx->grid.W);
    ctx->smem_coarse = (size_t)ctx->MW * sizeof(uint32_t) + (size_t)2 * m * sizeof(float);
    if (ctx->smem > 232448 || ctx->smem_coarse > 232448)
        return fail(ctx, AM_EINVAL, "grid %dx%d needs %zu B of shared memory per CTA: too large", m,
                    ctx->grid.n, ctx->smem);
    CK(cudaFuncSetAttribute(row_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ctx->smem));
    CK(cudaFuncSetAttribute(row_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ctx->smem));
    ctx->smem_cmap = clear_map_smem_bytes(ctx->MW);
    CK(cudaFuncSetAttribute(clear_map_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ctx->smem_cmap));
    int occ = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, filter_kernel, kThreads, 0);
    if (e != cudaSuccess || occ < 1) {
        cudaGetLastError();
        return fail(ctx, AM_EINVAL, "grid %dx%d needs %zu B of shared memory per CTA: too large", m,
                    ctx->grid.n, ctx->smem);
    }
    ctx->occ = occ;
    // the TMA-staged full-stream filter (one ring shape per AM_OPT_STREAM_TMA value)
    for (int k = 1; k <= kTmaShapes; ++k) {
        ctx->occ_tma[k] = 0;
        const void* fn = tma_kernel(k);
        const size_t sm = tma_smem(k);
        if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm) != cudaSuccess ||
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ctx->occ_tma[k], fn, tma_threads(k), sm) != cudaSuccess)
            ctx->occ_tma[k] = 0;
    }
    cudaGetLastError();
    // the fused pipeline: all CTAs co-resident (cooperative launch)
    ctx->smem_fused = fused_smem_bytes(m, ctx->grid.W);
    ctx->fused_grid = 0;
    if (ctx->smem_fused <= 232448 &&
        cudaFuncSetAttribute(am_pipeline_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)ctx->smem_fused) == cudaSuccess &&
        cudaFuncSetAttribute(am_pipeline_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)ctx->smem_fused) == cudaSuccess) {
        int occf = 0, occb = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occf, am_pipeline_kernel<false>, kThreads,
                                                          ctx->smem_fused) == cudaSuccess &&
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occb, am_pipeline_kernel<true>, kThreads,
                                                          ctx->smem_fused) == cudaSuccess &&
            occf > 0 && occb > 0)
            ctx->fused_grid = std::min(occf, occb) * ctx->sms;
        int occl = 0;
        if (cudaFuncSetAttribute(am_latency_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)ctx->smem_fused) == cudaSuccess &&
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occl, am_latency_kernel, kThreads, ctx->smem_fused) ==
                cudaSuccess &&
            occl > 0)
            ctx->lat_grid = occl * ctx->sms;
    }
    cudaGetLastError();
    // batched phases (batch.cuh)
    const int sm_rows = (int)((ctx->MW + ((m + 31) >> 5) + 1) * sizeof(uint32_t));
    CK(cudaFuncSetAttribute(bk_cones<BK_L0>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm_rows));
    CK(cudaFuncSetAttribute(bk_cones<BK_L1>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm_rows));
    CK(cudaFuncSetAttribute(bk_cones<BK_LIVE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ctx->smem_fused));
    CK(cudaFuncSetAttribute(bk_rows<BK_L0>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm_rows));
    CK(cudaFuncSetAttribute(bk_rows<BK_L1>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm_rows));
    CK(cudaFuncSetAttribute(bk_rows<BK_LIVE>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm_rows));
    CK(cudaFuncSetAttribute(bk_map<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ctx->smem_fused));
    CK(cudaFuncSetAttribute(bk_map<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ctx->smem_fused));
    CK(cudaFuncSetAttribute(bk_level0, cudaFuncAttributeMaxDynamicSharedMemorySize, sm_rows));
    CK(cudaFuncSetAttribute(bk_level1, cudaFuncAttributeMaxDynamicSharedMemorySize, sm_rows));
    CK(cudaFuncSetAttribute(bk_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ctx->smem_fused));
    return AM_OK;
}

// cone_kernel then row_kernel over the live list of p (stage s: its counters).
int launch_cones_rows(am_ctx* ctx, StreamParams p, bool coarse, int stage, cudaStream_t s) {
    p.recs = ctx->d_recs;
    p.tasks = ctx->d_tasks;
    p.rec_count = reinterpret_cast<unsigned int*>(ctx->d_ctr + kCtrRT + 2 * stage);
    p.task_count = ctx->d_ctr + kCtrRT + 2 * stage + 1;
    p.rec_cap = kRecCap;
    p.task_cap = kTaskCap;
    const unsigned int gc = (unsigned int)(ctx->sms * 8);
    const unsigned int gr = (unsigned int)(ctx->sms * kLiveBlocksPerSM);
    int rc;
    if (coarse) {
        cone_kernel<true><<<gc, kThreads, 0, s>>>(p);
        if ((rc = kmark(ctx, s, stage == 0 ? AM_K_L0_CONES : AM_K_L1_CONES))) return rc;
        row_kernel<true><<<gr, kThreads, ctx->smem, s>>>(p);
        if ((rc = kmark(ctx, s, stage == 0 ? AM_K_L0_ROWS : AM_K_L1_ROWS))) return rc;
    } else {
        cone_kernel<false><<<gc, kThreads, 0, s>>>(p);
        if ((rc = kmark(ctx, s, AM_K_LIVE_CONES))) return rc;
        row_kernel<false><<<gr, kThreads, ctx->smem, s>>>(p);
        if ((rc = kmark(ctx, s, AM_K_LIVE_ROWS))) return rc;
    }
    return AM_OK;
}

// The full voxel stream over vox[0, n) with clear-direction map `cmap`.
int launch_stream(am_ctx* ctx, StreamParams p, const float4* vox, long long n, const float4* cmap, bool timed,
                  cudaStream_t s, bool coarse = false) {
    if (n <= 0) return AM_OK;
    p.vox = vox;
    p.N = n;
    p.vbase = 0;
    p.vtag = 0;
    p.cmap = cmap;
    p.live_count = reinterpret_cast<unsigned int*>(ctx->d_ctr + kCtrTiles + (coarse ? 4 : 0));
    if (coarse) p.stats = ctx->d_ctr + kCtrWords;  // keep am_stats about the full stream
    p.live_idx = ctx->d_live_full;
    const long long ntiles = (n + kTile - 1) / kTile;
    long long g = ctx->grid_ctas > 0 ? ctx->grid_ctas : (long long)ctx->sms * ctx->occ;
    if (g > ntiles) g = ntiles;
    if (g < 1) g = 1;
    timed = timed && ctx->timing;
    if (timed) {
        if (ctx->ev_used == ctx->ev_start.size()) {
            cudaEvent_t a, b;
            CK(cudaEventCreate(&a));
            CK(cudaEventCreate(&b));
            ctx->ev_start.push_back(a);
            ctx->ev_stop.push_back(b);
        }
        CK(cudaEventRecord(ctx->ev_start[ctx->ev_used], s));
    }
    if (!coarse && ctx->bricks_on && ctx->d_bricks) {
        p.bricks = ctx->d_bricks;
        p.nbricks = ctx->nbricks;
        p.brick_list = ctx->d_brick_list;
        p.brick_count = reinterpret_cast<unsigned int*>(ctx->d_ctr + kCtrBricks);
        long long gb = ((long long)ctx->nbricks + kThreads - 1) / kThreads;
        const long long gmax = ctx->grid_ctas > 0 ? ctx->grid_ctas : (long long)ctx->sms * 8;
        if (gb > gmax) gb = gmax;
        if (gb < 1) gb = 1;
        brick_test_kernel<<<(unsigned)gb, kThreads, 0, s>>>(p);
        int rc;
        if ((rc = kmark(ctx, s, AM_K_BRICKS))) return rc;
        brick_voxels_kernel<<<(unsigned)gmax, kThreads, 0, s>>>(p);
        if ((rc = kmark(ctx, s, AM_K_VOXELS))) return rc;
    } else if (ctx->stream_tma && ctx->occ_tma[ctx->stream_tma] > 0) {
        const int k = ctx->stream_tma;
        const long long tiles = (n + tma_tile_vox(k) - 1) / tma_tile_vox(k);
        long long gt = ctx->grid_ctas > 0 ? ctx->grid_ctas : (long long)ctx->sms * ctx->occ_tma[k];
        if (gt > tiles) gt = tiles;
        if (gt < 1) gt = 1;
        void* args[] = {&p};
        CK(cudaLaunchKernel(tma_kernel(k), dim3((unsigned)gt), dim3(tma_threads(k)), args, tma_smem(k), s));
        int rc;
        if ((rc = kmark(ctx, s, AM_K_FILTER))) return rc;
    } else {
        filter_kernel<<<(unsigned)g, kThreads, 0, s>>>(p);
        int rc;
        if ((rc = kmark(ctx, s, AM_K_FILTER))) return rc;
    }
    if (timed) CK(cudaEventRecord(ctx->ev_stop[ctx->ev_used++], s));
    return launch_cones_rows(ctx, p, coarse, coarse ? 1 : 2, s);
}

// A coarse level: inner cones of every voxel of vox[0, n) (no filter).
int launch_coarse(am_ctx* ctx, StreamParams p, const float4* vox, long long n, const float4* cmap, int stage,
                  cudaStream_t s) {
    if (n <= 0) return AM_OK;
    p.vox = vox;
    p.N = n;
    p.cmap = cmap;
    p.live_idx = nullptr;  // every voxel of the level is live
    p.live_count = nullptr;
    p.stats = ctx->d_ctr + kCtrWords;  // keep am_stats about the full stream
    return launch_cones_rows(ctx, p, true, stage, s);
}

// Clear-direction map from `gam` into d_cmap (slot 0).
int launch_clear_map(am_ctx* ctx, const uint32_t* gam, cudaStream_t s) {
    const int ntex = 6 * ctx->cmapT * ctx->cmapT;
    const int gcm = std::max(1, std::min(ctx->sms * 4, (ntex / 16 + 7) / 8));
    clear_map_kernel<<<gcm, 256, ctx->smem_cmap, s>>>(gam, ctx->grid, ctx->d_tab, ctx->d_texels, ctx->cmapT,
                                                      ctx->d_cmap, ctx->d_ctr + 1 + ST_EARLY);
    return kmark(ctx, s, AM_K_CLEAR_MAP);
}

// One AICA map into device buffer gam (asynchronous on s):
//   level 0 (largest voxels, inner cones, one warp each) -> clear map ->
//   level 1 (next largest + strided sample, filtered, inner cones) -> clear map
//   -> the full stream of every voxel, filtered by the map, both cones ->
//   deferred band.  The coarse levels only make the filter effective; they are
//   subsets of the model, so the map is the same with any number of them
//   (AM_OPT_PHASES = 0, 1 or 2 levels).
// Can the whole map run as one fused cooperative launch?
// Small models (latency.cuh): level 0 is the whole model, no clear-direction maps or bricks.
bool small_model(const am_ctx* ctx) { return ctx->N <= kSmallModel || ctx->n_l0 == 0; }

bool fused_ok(const am_ctx* ctx) {
    return ctx->fused && ctx->fused_grid > 0 && !(ctx->diag & 3) && ctx->N > 0 &&
           (small_model(ctx) || (ctx->phases >= 1 && ctx->n_l0 > 0 && ctx->bricks_on && ctx->d_bricks));
}

// The fused launch parameters for slot 0 and the map gam.
FusedParams fused_params(am_ctx* ctx, const float* pivot, uint32_t* gam) {
    FusedParams F{};
    F.main = make_params(ctx, pivot, gam);
    F.main.vox = ctx->d_vox;
    F.main.N = ctx->N;
    F.main.cmap = ctx->d_cmap;
    F.main.bricks = ctx->d_bricks;
    F.main.nbricks = ctx->nbricks;
    F.main.subs = (ctx->subs_on & 1) ? ctx->d_subs : nullptr;
    F.main.supers = (ctx->subs_on & 2) ? ctx->d_supers : nullptr;
    F.main.super_list = ctx->d_brick_list + 8ull * ctx->nbricks;
    F.main.super_count = reinterpret_cast<unsigned int*>(ctx->d_ctr + kCtrSupers);
    F.main.brick_list = ctx->d_brick_list;
    F.main.brick_count = reinterpret_cast<unsigned int*>(ctx->d_ctr + kCtrBricks);
    F.main.recs = ctx->d_recs;
    F.main.tasks = ctx->d_tasks;
    F.main.rec_count = reinterpret_cast<unsigned int*>(ctx->d_ctr + kCtrRT + 4);
    F.main.task_count = ctx->d_ctr + kCtrRT + 5;
    F.main.rec_cap = kRecCap;
    F.main.task_cap = kTaskCap;
    F.main.live_count = reinterpret_cast<unsigned int*>(ctx->d_ctr + kCtrTiles);
    F.main.live_idx = ctx->d_live_full;  // (single pivot; launch_batch_layers / launch_fused_batch: d_live)
    F.lvl = F.main;
    F.lvl.vox = ctx->d_coarse;
    F.lvl.N = ctx->n_l0;
    F.lvl.cmap = ctx->d_cmap_ones;
    F.lvl.stats = ctx->d_ctr + kCtrWords;
    F.lvl.rec_count = reinterpret_cast<unsigned int*>(ctx->d_ctr + kCtrRT);
    F.lvl.task_count = ctx->d_ctr + kCtrRT + 1;
    F.lvl.rec_cap = kRecCap / 2;
    F.lvl.task_cap = kTaskCap / 2;
    F.l1 = ctx->d_coarse + ctx->n_l0;
    F.l1subs = ctx->l1_subs ? ctx->d_l1subs : nullptr;
    F.clear1 = ctx->l1_sparse > 0 ? ctx->d_ctr + kCtrClear1 : nullptr;
    F.l1_sparse = ctx->l1_sparse;
    F.n0 = (unsigned int)ctx->n_l0;
    F.n1 = (unsigned int)(ctx->n_l1 - ctx->n_l0);
    F.rec1 = reinterpret_cast<unsigned int*>(ctx->d_ctr + kCtrRT + 2);
    F.task1 = ctx->d_ctr + kCtrRT + 3;
    F.live1 = nullptr;
    F.texels = ctx->d_texels;
    F.ntex = 6 * ctx->cmapT * ctx->cmapT;
    F.texels1 = ctx->d_texels1;
    F.cmapT1 = ctx->cmapT1;
    F.use_l1 = ctx->phases == 2;
    F.ts = (ctx->diag_ts && ctx->d_ts) ? ctx->d_ts : nullptr;  // batched: group 0
    return F;
}

int timed_begin(am_ctx* ctx, cudaStream_t s) {
    if (!ctx->timing) return AM_OK;
    if (ctx->ev_used == ctx->ev_start.size()) {
        cudaEvent_t a, b;
        CK(cudaEventCreate(&a));
        CK(cudaEventCreate(&b));
        ctx->ev_start.push_back(a);
        ctx->ev_stop.push_back(b);
    }
    CK(cudaEventRecord(ctx->ev_start[ctx->ev_used], s));
    return AM_OK;
}

int timed_end(am_ctx* ctx, cudaStream_t s) {
    if (ctx->timing) CK(cudaEventRecord(ctx->ev_stop[ctx->ev_used++], s));
    return AM_OK;
}

// Per-kernel accounting.  kchain(): start a chain of launches on s (records an
// event when timing per kernel).  kmark(k): one launch of kernel k just went
// onto s -- counts it and, when timing per kernel, records the event that ends
// it (the previous event of the chain starts it; launches on one stream run in
// order, so the interval is that kernel's device time plus the gap between).
int kpool_event(am_ctx* ctx, size_t* idx) {
    if (ctx->kev_used == ctx->kev.size()) {
        cudaEvent_t e;
        CK(cudaEventCreate(&e));
        ctx->kev.push_back(e);
    }
    *idx = ctx->kev_used++;
    return AM_OK;
}

int kchain(am_ctx* ctx, cudaStream_t s) {
    ctx->kev_prev = -1;
    if (ctx->timing != 2) return AM_OK;
    size_t i;
    int rc = kpool_event(ctx, &i);
    if (rc) return rc;
    CK(cudaEventRecord(ctx->kev[i], s));
    ctx->kev_prev = (long long)i;
    return AM_OK;
}

int kmark(am_ctx* ctx, cudaStream_t s, int k) {
    CK(cudaGetLastError());
    ctx->k_launches[k] += 1;
    if (ctx->timing != 2 || ctx->kev_prev < 0) return AM_OK;
    size_t i;
    int rc = kpool_event(ctx, &i);
    if (rc) return rc;
    CK(cudaEventRecord(ctx->kev[i], s));
    ctx->kmarks.emplace_back(k, i);
    ctx->kmark_begin.push_back((size_t)ctx->kev_prev);
    ctx->kev_prev = (long long)i;
    return AM_OK;
}

// One map (pivot) into gam with one fused cooperative launch over the whole grid.
int launch_fused(am_ctx* ctx, const float* pivot, uint32_t* gam, cudaStream_t s) {
    const bool lat = ctx->lat_grid > 0 && !(ctx->diag & 16);
    CK(cudaMemsetAsync(gam, 0, (size_t)ctx->MW * sizeof(uint32_t), s));
    if (!lat) CK(cudaMemsetAsync(ctx->d_ctr, 0, kCtrStride * sizeof(unsigned long long), s));
    FusedParams F = fused_params(ctx, pivot, gam);
    F.ctr0 = ctx->d_ctr;  // (am_latency_kernel zeroes the map's counters itself)
    F.ctr_words = kCtrStride;
    if (small_model(ctx)) {  // level 0 = every voxel; the all-clear map (no map is built)
        F.small = 1;
        F.lvl.vox = ctx->d_vox;
        F.lvl.N = ctx->N;
        F.n0 = (unsigned int)ctx->N;
        F.n1 = 0;
        F.use_l1 = 0;
        F.main.cmap = ctx->d_cmap_ones;
    }
    int rc;
    if ((rc = timed_begin(ctx, s))) return rc;
    if ((rc = kchain(ctx, s))) return rc;
    void* args[] = {&F};
    if (lat) {
        CK(cudaLaunchCooperativeKernel((const void*)am_latency_kernel, dim3(ctx->lat_grid), dim3(kThreads), args,
                                       ctx->smem_fused, s));
    } else {  // (AM_OPT_DIAG bit 4: the previous single-pivot kernel, for comparison)
        F.small = 0;
        CK(cudaLaunchCooperativeKernel((const void*)am_pipeline_kernel<false>, dim3(ctx->fused_grid), dim3(kThreads),
                                       args, ctx->smem_fused, s));
    }
    if ((rc = kmark(ctx, s, AM_K_FUSED))) return rc;
    if ((rc = timed_end(ctx, s))) return rc;
    if (ctx->d_prev)
        CK(cudaMemcpyAsync(ctx->d_prev, gam, (size_t)ctx->MW * sizeof(uint32_t), cudaMemcpyDeviceToDevice, s));
    return AM_OK;
}

// The batch's pivots (xyz + may_cull) into ctx->d_piv, from pinned host staging
// (the async copy of the previous call is waited for before the staging is rewritten).
int upload_pivots(am_ctx* ctx, const float* pivots, int64_t P, uint32_t* gam0, cudaStream_t s) {
    if (!ctx->piv_ev) CK(cudaEventCreateWithFlags(&ctx->piv_ev, cudaEventDisableTiming));
    CK(cudaEventSynchronize(ctx->piv_ev));
    if (ctx->h_piv_cap < P + 1) {
        if (ctx->h_piv) cudaFreeHost(ctx->h_piv);
        ctx->h_piv = nullptr;
        ctx->h_piv_cap = 0;
        CK(cudaMallocHost(&ctx->h_piv, (size_t)(P + 1) * sizeof(float4)));
        ctx->h_piv_cap = P + 1;
    }
    for (int64_t k = 0; k < P; ++k) {
        const StreamParams pk = make_params(ctx, pivots + 3 * k, gam0);
        ctx->h_piv[k] = make_float4(pk.px, pk.py, pk.pz, pk.may_cull ? 1.f : 0.f);
    }
    // entry P: the output base of the call (read by the batched kernels: a captured chain replays
    // into any output buffer)
    const unsigned long long outp = (unsigned long long)(uintptr_t)gam0;
    std::memset(&ctx->h_piv[P], 0, sizeof(float4));
    std::memcpy(&ctx->h_piv[P], &outp, sizeof outp);
    std::memcpy(reinterpret_cast<char*>(&ctx->h_piv[P]) + 8, &ctx->reuse_parity, sizeof(unsigned int));
    CK(cudaMemcpyAsync(ctx->d_piv, ctx->h_piv, (size_t)(P + 1) * sizeof(float4), cudaMemcpyHostToDevice, s));
    CK(cudaEventRecord(ctx->piv_ev, s));
    return AM_OK;
}

// P maps (pivots[3P]) into gam0 + k * MW with ONE fused launch: K groups of
// CTAs (K <= ctx->slots) take pivots from a device queue (fused.cuh).
int ensure_piv(am_ctx* ctx, int64_t P) {
    if (ctx->piv_cap >= P + 1) return AM_OK;
    ++ctx->gen;
    cudaFree(ctx->d_piv);
    ctx->d_piv = nullptr;
    ctx->piv_cap = 0;
    CK(cudaMalloc(&ctx->d_piv, (size_t)(P + 1) * sizeof(float4)));
    ctx->piv_cap = P + 1;
    return AM_OK;
}

int launch_fused_batch(am_ctx* ctx, const float* pivots, int64_t P, int K, uint32_t* gam0, cudaStream_t s) {
    {
        int rc;
        if ((rc = ensure_piv(ctx, P)) != AM_OK) return rc;
    }
    if (!ctx->d_bctl) CK(cudaMalloc(&ctx->d_bctl, kBctlWords * sizeof(unsigned long long)));
    {
        int rc;
        if ((rc = upload_pivots(ctx, pivots, P, gam0, s)) != AM_OK) return rc;
    }
    CK(cudaMemsetAsync(ctx->d_bctl, 0, kBctlWords * sizeof(unsigned long long), s));
    FusedParams F = fused_params(ctx, pivots, gam0);
    const int ntex = 6 * ctx->cmapT * ctx->cmapT;
    F.nslot = K;
    F.ctr_stride = (unsigned long long)kCtrStride * sizeof(unsigned long long);
    F.q_stride = (unsigned long long)ctx->qcap * sizeof(unsigned long long);
    F.rec_stride = (unsigned long long)kRecCap * sizeof(ConeRec);
    F.task_stride = (unsigned long long)kTaskCap * sizeof(unsigned long long);
    F.live_stride = (unsigned long long)ctx->live_cap * sizeof(unsigned int);
    F.main.live_idx = ctx->d_live;
    F.main.live_cap = (unsigned int)ctx->live_cap;
    F.cmap_stride = (unsigned long long)ntex * sizeof(float4);
    F.blist_stride = blist_words(ctx) * sizeof(unsigned int);
    F.piv = ctx->d_piv;
    F.npiv = (unsigned int)P;
    F.gam0 = gam0;
    F.ctr0 = ctx->d_ctr;
    F.ctr_words = kCtrStride;
    F.bar = ctx->d_bctl;                                             // 2 words per group
    F.qnext = reinterpret_cast<unsigned int*>(ctx->d_bctl + 2 * kMaxSlots);
    F.cur = F.qnext + 1;                                             // kMaxSlots words
    int rc;
    if ((rc = timed_begin(ctx, s))) return rc;
    if ((rc = kchain(ctx, s))) return rc;
    void* args[] = {&F};
    CK(cudaLaunchCooperativeKernel((const void*)am_pipeline_kernel<true>, dim3(ctx->fused_grid), dim3(kThreads), args,
                                   ctx->smem_fused, s));
    if ((rc = kmark(ctx, s, AM_K_FUSED))) return rc;
    return timed_end(ctx, s);
}

// P maps (pivots[3P]) into gam0 + k * MW, phase by phase over chunks of up to
// ctx->batch pivots (batch.cuh): each phase is one launch with blockIdx.y =
// pivot of the chunk.
// Host mirror of fused.cuh slot_params for a whole launch: advance the slot-0
// per-map pointers of F by `base` slots, so that launch pivot y uses slot base + y.
template <typename T>
T* hshift(T* p, unsigned long long b) {
    return p ? reinterpret_cast<T*>(reinterpret_cast<uintptr_t>(p) + b) : p;
}

void shift_slots(FusedParams& F, int base) {
    if (base == 0) return;
    const unsigned long long b = (unsigned long long)base;
    for (int which = 0; which < 2; ++which) {
        StreamParams& p = which ? F.lvl : F.main;
        p.qcount = hshift(p.qcount, b * F.ctr_stride);
        p.stats = hshift(p.stats, b * F.ctr_stride);
        p.early = hshift(p.early, b * F.ctr_stride);
        p.live_count = hshift(p.live_count, b * F.ctr_stride);
        p.rec_count = hshift(p.rec_count, b * F.ctr_stride);
        p.task_count = hshift(p.task_count, b * F.ctr_stride);
        p.brick_count = hshift(p.brick_count, b * F.ctr_stride);
        p.queue = hshift(p.queue, b * F.q_stride);
        p.live_idx = hshift(p.live_idx, b * F.live_stride);
        p.recs = hshift(p.recs, b * F.rec_stride);
        p.tasks = hshift(p.tasks, b * F.task_stride);
        p.brick_list = hshift(p.brick_list, b * F.blist_stride);
        p.super_list = hshift(p.super_list, b * F.blist_stride);
        p.super_count = hshift(p.super_count, b * F.ctr_stride);
        if (!which) p.cmap = hshift(p.cmap, b * F.cmap_stride);
    }
    F.rec1 = hshift(F.rec1, b * F.ctr_stride);
    F.task1 = hshift(F.task1, b * F.ctr_stride);
    F.ctr0 = hshift(F.ctr0, b * F.ctr_stride);
    if (F.wit0) {
        F.wit0 += b * 2 * (unsigned long long)F.main.grid.m * F.main.grid.n;
        F.hash0 += b * F.hash_words;
    }
}

// Streams (and fork/join events) of the batched path's lanes.
int ensure_lanes(am_ctx* ctx, int lanes) {
    for (int l = 0; l < lanes; ++l)
        if (!ctx->lane_s[l]) CK(cudaStreamCreateWithFlags(&ctx->lane_s[l], cudaStreamNonBlocking));
    for (int l = 0; l <= kMaxLanes; ++l)
        if (!ctx->lane_ev[l]) CK(cudaEventCreateWithFlags(&ctx->lane_ev[l], cudaEventDisableTiming));
    return AM_OK;
}

int launch_batch_layers(am_ctx* ctx, const float* pivots, int64_t P, uint32_t* gam0, cudaStream_t s) {
    const int K = (int)std::min<int64_t>(P, ctx->batch);
    int rc;
    if ((rc = ensure_slots(ctx, K)) != AM_OK) return rc;
    if ((rc = ensure_piv(ctx, P)) != AM_OK) return rc;
    const size_t mn = (size_t)ctx->grid.m * ctx->grid.n;
    if (ctx->reuse && ctx->contrib_slots < ctx->slots) {  // AM_OPT_REUSE witness arrays (no witness at first)
        cudaFree(ctx->d_wit);
        cudaFree(ctx->d_hash);
        ctx->d_wit = nullptr;
        ctx->d_hash = nullptr;
        ctx->contrib_slots = 0;
        unsigned int hw = 1;
        while (hw < 2 * mn) hw <<= 1;
        CK(cudaMalloc(&ctx->d_wit, (size_t)ctx->slots * 2 * mn * sizeof(unsigned int)));
        CK(cudaMalloc(&ctx->d_hash, (size_t)ctx->slots * hw * sizeof(unsigned int)));
        CK(cudaMemset(ctx->d_wit, 0xff, (size_t)ctx->slots * 2 * mn * sizeof(unsigned int)));
        ctx->hash_words = hw;
        ctx->contrib_slots = ctx->slots;
        ++ctx->gen;
    }
    {
        int rc;
        if ((rc = upload_pivots(ctx, pivots, P, gam0, s)) != AM_OK) return rc;
    }
    if (ctx->reuse) ctx->reuse_parity ^= 1u;  // (the next call reads what this one writes)
    const int ntex = 6 * ctx->cmapT * ctx->cmapT;
    const size_t sm_rows = (size_t)(ctx->MW + ((ctx->grid.m + 31) >> 5) + 1) * sizeof(uint32_t);
    // one chunk of kk pivots from c0 on, slots [sb, sb + kk), on stream s
    auto run_chunk = [&](int64_t c0, int kk, int sb, cudaStream_t s) -> int {
        int rc;
        uint32_t* g = gam0 + c0 * ctx->MW;
        FusedParams F = fused_params(ctx, pivots + 3 * c0, g);
        F.out_ptr = reinterpret_cast<const unsigned long long*>(ctx->d_piv + P);  // the call's output base
        F.out_off = (unsigned long long)c0 * ctx->MW;
        if (ctx->reuse) {
            F.wit0 = ctx->d_wit;
            F.hash0 = ctx->d_hash;
            F.hash_words = ctx->hash_words;
        }
        F.nslot = kk;
        F.ctr_stride = (unsigned long long)kCtrStride * sizeof(unsigned long long);
        F.q_stride = (unsigned long long)ctx->qcap * sizeof(unsigned long long);
        F.rec_stride = (unsigned long long)kRecCap * sizeof(ConeRec);
        F.task_stride = (unsigned long long)kTaskCap * sizeof(unsigned long long);
        F.live_stride = (unsigned long long)ctx->live_cap * sizeof(unsigned int);
        F.main.live_idx = ctx->d_live;  // (the slots' capped lists; an overflow is re-streamed: live_overflow_rescan)
        F.main.live_cap = (unsigned int)ctx->live_cap;
        F.cmap_stride = (unsigned long long)ntex * sizeof(float4);
        F.blist_stride = blist_words(ctx) * sizeof(unsigned int);
        F.piv = ctx->d_piv + c0;
        F.npiv = (unsigned int)kk;
        F.gam0 = g;
        F.ctr0 = ctx->d_ctr;
        F.ctr_words = kCtrStride;
        shift_slots(F, sb);
        if ((rc = kchain(ctx, s))) return rc;
        auto grid = [&](long long items, long long per_cta, int cap) {
            long long gx = (items + per_cta - 1) / per_cta;
            return dim3((unsigned)std::max<long long>(1, std::min<long long>(gx, cap)), (unsigned)kk);
        };
        const dim3 b(kThreads);
        const int map_cap = ctx->bk_map_ctas > 0 ? ctx->bk_map_ctas : (1 << 16);
#define AM_KM(k) if ((rc = kmark(ctx, s, k))) return rc
        // (AM_OPT_PDL: programmatic stream serialisation -- the kernel's CTAs may start under the previous
        //  kernel's tail and run their parameter prologue there; batch.cuh grid_dep_wait orders the rest)
        auto L = [&](auto kern, dim3 g, size_t smem, dim3 bd = dim3(kThreads)) -> int {
            if (ctx->pdl) {
                cudaLaunchConfig_t lc{};
                lc.gridDim = g;
                lc.blockDim = bd;
                lc.dynamicSmemBytes = smem;
                lc.stream = s;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
                at[0].val.programmaticStreamSerializationAllowed = 1;
                lc.attrs = at;
                lc.numAttrs = 1;
                CK(cudaLaunchKernelEx(&lc, kern, F));
            } else {
                kern<<<g, bd, smem, s>>>(F);
            }
            return AM_OK;
        };
        bk_init<<<kk, b, 0, s>>>(F);  // this chunk's maps and counters start at zero
        AM_KM(AM_K_INIT);
        const long long n0e = ctx->n_l0 + (ctx->reuse ? ctx->grid.m * ctx->grid.n : 0);  // (+ reuse witnesses)
        if (ctx->stage_fusion & 1) {
            // (AM + row-full bits only; AM_L0_PER_CTA level-0 voxels per CTA, their rows shared by its 256 threads)
            if ((rc = L(bk_level0, grid(n0e, AM_L0_PER_CTA, AM_L0_CTAS), sm_rows))) return rc;
            AM_KM(AM_K_LEVEL0);
        } else {
            if ((rc = L(bk_cones<BK_L0>, grid(n0e, kThreads, 1 << 16), sm_rows))) return rc;
            AM_KM(AM_K_L0_CONES);
            if ((rc = L(bk_rows<BK_L0>, grid(1 << 30, 1, ctx->bk_rows_ctas), sm_rows))) return rc;
            AM_KM(AM_K_L0_ROWS);
        }
        if (F.use_l1) {
            // (few texels, many clear cells after level 0: spread them over more CTAs -- one
            // warp per 4 x 4 coarse texel on the coarse-block path)
            const long long nt1 = 6ll * ctx->cmapT1 * ctx->cmapT1;
            // (AM_MAP1_WARP_TEXEL: one warp per texel, <= 4 texels per warp -- clear_map_cta's warp_texel path)
            const long long g1 = AM_MAP1_WARP_TEXEL
                                     ? (nt1 + 4 * (kThreads / 32) - 1) / (4 * (kThreads / 32))
                                     : std::max(nt1 / (4 * kThreads), nt1 / ((AM_MAP1_BLOCK4 ? 16 : 64) * AM_MAP1_WARP_BLOCKS / 4 * (kThreads / 32)));
            if ((rc = L(bk_map<true>, grid(std::max(1ll, g1), 1, 1 << 16), ctx->smem_fused))) return rc;
        } else {
            if ((rc = L(bk_map<false>, grid(ntex, 4 * kThreads, map_cap), ctx->smem_fused))) return rc;
        }
        AM_KM(AM_K_CLEAR_MAP);
        if (F.use_l1) {
            if (ctx->stage_fusion & 2) {
                if ((rc = L(bk_level1, grid(ctx->n_l1 - ctx->n_l0, kThreads, ctx->bk_cone_ctas), sm_rows)))
                    return rc;
                AM_KM(AM_K_LEVEL1);
            } else {
                if ((rc = L(bk_cones<BK_L1>, grid(ctx->n_l1 - ctx->n_l0, AM_L1_STEPS * kThreads, 1 << 16), sm_rows)))
                    return rc;
                AM_KM(AM_K_L1_CONES);
                if ((rc = L(bk_rows<BK_L1>, grid(1 << 30, 1, ctx->bk_rows_ctas), sm_rows))) return rc;
                AM_KM(AM_K_L1_ROWS);
            }
            if ((rc = L(bk_map<false>, grid(ntex, 4 * kThreads, map_cap), ctx->smem_fused))) return rc;
            AM_KM(AM_K_CLEAR_MAP);
        }
        if (F.main.supers && AM_FUSED_BRICKS) {  // super-bricks -> bricks -> sub-bricks in one launch
            if ((rc = L(bk_bricks_fused, grid((ctx->nbricks + 7) / 8, AM_FUSED_BRICKS_SUPERS, 1 << 16), 0))) return rc;
            AM_KM(AM_K_BRICKS);
        } else {
            if (F.main.supers) {
                if ((rc = L(bk_supers, grid((ctx->nbricks + 7) / 8, AM_BRICK_STEPS * kThreads, 1 << 16), 0))) return rc;
                AM_KM(AM_K_BRICKS);
            }
            if ((rc = L(bk_bricks, grid(ctx->nbricks, AM_BRICK_STEPS * kThreads, F.main.supers ? AM_BRICKS_CTAS : (1 << 16)), 0)))
                return rc;
            AM_KM(AM_K_BRICKS);
        }
        if (ctx->stage_fusion & 4) {
            if ((rc = L(bk_stream, grid(1 << 30, 1, ctx->bk_voxel_ctas), ctx->smem_fused))) return rc;
            AM_KM(AM_K_STREAM);
        } else {
            if ((rc = L(bk_voxels, grid(1 << 30, 1, ctx->bk_voxel_ctas), 0))) return rc;
            AM_KM(AM_K_VOXELS);
            if ((rc = L(bk_cones<BK_LIVE>, grid(1 << 30, 1, ctx->bk_cone_ctas), ctx->smem_fused))) return rc;
            AM_KM(AM_K_LIVE_CONES);
            if ((rc = L(bk_rows<BK_LIVE>, grid(1 << 30, 1, ctx->bk_rows_ctas), sm_rows))) return rc;
            AM_KM(AM_K_LIVE_ROWS);
        }
        // (few pairs, each a long exact test: small CTAs spread them over the SMs)
        if ((rc = L(bk_band, grid(1 << 30, 1, AM_BAND_CTAS), 0, dim3(AM_BAND_THREADS)))) return rc;
        AM_KM(AM_K_BAND);
#undef AM_KM
        return AM_OK;
    };
    // chunks of Kl pivots round-robin over `lanes` streams, lane l on slots
    // [l Kl, (l + 1) Kl): one lane's phase tails overlap another's launches
    // (per-kernel timing keeps one stream so its events bracket single kernels)
    const int lanes = ctx->timing == 2 ? 1 : (int)std::max<int64_t>(1, std::min<int64_t>(ctx->lanes, K));
    const int Kl = K / lanes;  // (lanes <= K: lane slots stay inside the K allocated)
    auto chain = [&](cudaStream_t cs) -> int {
        int rc;
        if (lanes == 1) {
            for (int64_t c0 = 0; c0 < P; c0 += K)
                if ((rc = run_chunk(c0, (int)std::min<int64_t>(K, P - c0), 0, cs))) return rc;
            return AM_OK;
        }
        if ((rc = ensure_lanes(ctx, lanes))) return rc;
        CK(cudaEventRecord(ctx->lane_ev[lanes], cs));
        for (int l = 0; l < lanes; ++l) CK(cudaStreamWaitEvent(ctx->lane_s[l], ctx->lane_ev[lanes], 0));
        int64_t chunk = 0;
        for (int64_t c0 = 0; c0 < P; c0 += Kl, ++chunk) {
            const int l = (int)(chunk % lanes);
            if ((rc = run_chunk(c0, (int)std::min<int64_t>(Kl, P - c0), l * Kl, ctx->lane_s[l]))) return rc;
        }
        for (int l = 0; l < lanes; ++l) {
            CK(cudaEventRecord(ctx->lane_ev[l], ctx->lane_s[l]));
            CK(cudaStreamWaitEvent(cs, ctx->lane_ev[l], 0));
        }
        return AM_OK;
    };
    if ((rc = timed_begin(ctx, s))) return rc;
    // CUDA graph: the whole chain (memsets, ~11 launches per chunk, the lane fork /
    // join) captured once per (options, P, output, pivot buffer) and replayed: one
    // host call per batch instead of ~100 (not with per-kernel timing or diagnostics)
    if (ctx->use_graph && ctx->timing != 2 && ctx->diag == 0) {
        if (!(ctx->g_exec && ctx->g_gen == ctx->gen && ctx->g_P == P && ctx->g_piv == ctx->d_piv)) {
            if (ctx->g_exec) cudaGraphExecDestroy(ctx->g_exec);
            ctx->g_exec = nullptr;
            if (!ctx->cap_s) CK(cudaStreamCreateWithFlags(&ctx->cap_s, cudaStreamNonBlocking));
            long long before[AM_K_COUNT];
            std::copy(ctx->k_launches, ctx->k_launches + AM_K_COUNT, before);
            CK(cudaStreamBeginCapture(ctx->cap_s, cudaStreamCaptureModeThreadLocal));
            const int crc = chain(ctx->cap_s);
            cudaGraph_t graph = nullptr;
            const cudaError_t ce = cudaStreamEndCapture(ctx->cap_s, &graph);
            for (int k = 0; k < AM_K_COUNT; ++k) {  // the capture launched nothing
                ctx->g_launches[k] = ctx->k_launches[k] - before[k];
                ctx->k_launches[k] = before[k];
            }
            if (crc != AM_OK) {
                if (graph) cudaGraphDestroy(graph);
                return crc;
            }
            if (ce != cudaSuccess) return fail(ctx, AM_ECUDA, "graph capture: %s", cudaGetErrorString(ce));
            const cudaError_t ie = cudaGraphInstantiate(&ctx->g_exec, graph, 0);
            cudaGraphDestroy(graph);
            if (ie != cudaSuccess) {
                ctx->g_exec = nullptr;
                return fail(ctx, AM_ECUDA, "graph instantiate: %s", cudaGetErrorString(ie));
            }
            ctx->g_gen = ctx->gen;
            ctx->g_P = P;
            ctx->g_piv = ctx->d_piv;
        }
        CK(cudaGraphLaunch(ctx->g_exec, s));
        for (int k = 0; k < AM_K_COUNT; ++k) ctx->k_launches[k] += ctx->g_launches[k];
    } else {
        if ((rc = chain(s))) return rc;
    }
    return timed_end(ctx, s);
}

int launch_aica(am_ctx* ctx, const float pivot[3], uint32_t* gam, cudaStream_t s) {
    if (fused_ok(ctx)) return launch_fused(ctx, pivot, gam, s);
    CK(cudaMemsetAsync(gam, 0, (size_t)ctx->MW * sizeof(uint32_t), s));
    CK(cudaMemsetAsync(ctx->d_ctr, 0, kCtrStride * sizeof(unsigned long long), s));
    if (ctx->N == 0) return AM_OK;
    StreamParams p = make_params(ctx, pivot, gam);
    int rc;
    if ((rc = kchain(ctx, s))) return rc;
    const float4* cm = ctx->d_cmap_ones;
    if (ctx->diag & 2) {
        // diagnostic: clear map from the previous map computed on this context
        // (exact only when the previous call used the same pivot)
        CK(cudaMemcpyAsync(gam, ctx->d_prev, (size_t)ctx->MW * sizeof(uint32_t), cudaMemcpyDeviceToDevice, s));
        if ((rc = launch_clear_map(ctx, gam, s))) return rc;
        cm = ctx->d_cmap;
    } else if (ctx->phases > 0 && ctx->n_l0 > 0) {
        if ((rc = launch_coarse(ctx, p, ctx->d_coarse, ctx->n_l0, ctx->d_cmap_ones, 0, s))) return rc;
        if ((rc = launch_clear_map(ctx, gam, s))) return rc;
        if (ctx->phases > 1) {
            // level 1 through the same filter + live pipeline as the full stream
            // (inner cones only, no band)
            if ((rc = launch_stream(ctx, p, ctx->d_coarse + ctx->n_l0, ctx->n_l1 - ctx->n_l0, ctx->d_cmap, false, s,
                                    true)))
                return rc;
            if ((rc = launch_clear_map(ctx, gam, s))) return rc;
        }
        cm = ctx->d_cmap;
    }
    if (!(ctx->diag & 1)) {
        if ((rc = launch_stream(ctx, p, ctx->d_vox, ctx->N, cm, true, s))) return rc;
        band_exact_kernel<<<(unsigned)ctx->sms, kThreads, 0, s>>>(p);
        if ((rc = kmark(ctx, s, AM_K_BAND))) return rc;
    }
    if (ctx->d_prev)  // allocated once diagnostics were enabled
        CK(cudaMemcpyAsync(ctx->d_prev, gam, (size_t)ctx->MW * sizeof(uint32_t), cudaMemcpyDeviceToDevice, s));
    return AM_OK;
}

// Diagnostics (AM_OPT_DIAG bit 2): fused-phase end times (us) of the last
// launch on stderr (batched launches: group 0).
int print_phase_times(am_ctx* ctx) {
    if (!ctx->diag_ts || !ctx->d_ts) return AM_OK;
    unsigned long long t[16];
    CK(cudaMemcpy(t, ctx->d_ts, sizeof t, cudaMemcpyDeviceToHost));
    fprintf(stderr, "am fused phases (us):");
    for (int k = 1; k < 16; ++k)
        if (t[k] >= t[0] && t[k]) fprintf(stderr, " %d:%.1f", k, (t[k] - t[0]) * 1e-3);
    fprintf(stderr, "\n");
    CK(cudaMemset(ctx->d_ts, 0, sizeof t));
    // am_latency_kernel: per-CTA P6 end (us after the kernel start), live voxels, rows, filter survivors
    std::vector<unsigned long long> c(4 * kDiagCtas);
    CK(cudaMemcpy(c.data(), ctx->d_ts + 16, c.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost));
    std::vector<std::pair<double, int>> ends;
    for (int b = 0; b < kDiagCtas; ++b)
        if (c[4 * b] >= t[0] && c[4 * b]) ends.push_back({(c[4 * b] - t[0]) * 1e-3, b});
    if (!ends.empty()) {
        std::sort(ends.begin(), ends.end());
        const size_t nE = ends.size();
        fprintf(stderr, "am P6 per CTA (%zu): end us min %.1f med %.1f p90 %.1f max %.1f;", nE, ends[0].first,
                ends[nE / 2].first, ends[(nE * 9) / 10].first, ends[nE - 1].first);
        for (size_t k = nE >= 3 ? nE - 3 : 0; k < nE; ++k) {
            const int b = ends[k].second;
            fprintf(stderr, " cta %d: %.1f us live %llu rows %llu passed %llu;", b, ends[k].first, c[4 * b + 1],
                    c[4 * b + 2], c[4 * b + 3]);
        }
        unsigned long long lmax = 0, lsum = 0, rmax = 0, rsum = 0;
        for (auto& e : ends) {
            lmax = std::max(lmax, c[4 * e.second + 1]);
            lsum += c[4 * e.second + 1];
            rmax = std::max(rmax, c[4 * e.second + 2]);
            rsum += c[4 * e.second + 2];
        }
        fprintf(stderr, " live max %llu mean %.1f, rows max %llu mean %.1f\n", lmax, (double)lsum / nE, rmax,
                (double)rsum / nE);
        CK(cudaMemset(ctx->d_ts + 16, 0, c.size() * sizeof(unsigned long long)));
    }
    return AM_OK;
}

// Calls on one context share its scratch (per-map slots, pivots, host-output maps): a call on
// another stream than the previous one first waits for the previous call's end (done_ev).
int stream_begin(am_ctx* ctx, cudaStream_t s) {
    if (ctx->has_last && ctx->last_s != s) CK(cudaStreamWaitEvent(s, ctx->done_ev, 0));
    return AM_OK;
}

int stream_end(am_ctx* ctx, cudaStream_t s) {
    if (!ctx->done_ev) CK(cudaEventCreateWithFlags(&ctx->done_ev, cudaEventDisableTiming));
    CK(cudaEventRecord(ctx->done_ev, s));
    ctx->last_s = s;
    ctx->has_last = true;
    return AM_OK;
}

int check_pivot(am_ctx* ctx, const float* pivot) {
    if (!pivot) return fail(ctx, AM_EINVAL, "pivot is NULL");
    for (int k = 0; k < 3; ++k)
        if (!is_finite_f(pivot[k])) return fail(ctx, AM_EINVAL, "pivot[%d] is not finite", k);
    return AM_OK;
}

}  // namespace

extern "C" {

int am_create(const am_cylinder* tool, int n_cyl, int m, int n, int device, am_ctx** out) {
    if (!out) return AM_EINVAL;
    *out = nullptr;
    if (!tool || n_cyl < 1 || n_cyl > AM_MAX_CYL) return AM_EINVAL;
    if (m < 1 || m > 1024 || n < 1 || n > 1024) return AM_EINVAL;
    for (int k = 0; k < n_cyl; ++k) {
        if (!is_finite_f(tool[k].radius) || !is_finite_f(tool[k].height) || tool[k].radius <= 0.f ||
            tool[k].height <= 0.f)
            return AM_EINVAL;
    }
    am_ctx* ctx = new am_ctx();
    ctx->device = device;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
        cudaGetLastError();
        delete ctx;
        return AM_ECUDA;
    }
    DeviceGuard dg(device);
    if (!dg.ok) {
        delete ctx;
        return AM_ECUDA;
    }
    // tool: cylinders from the pivot outward (readings G3/G4); radii in double
    // then rounded, so the device sees the caller's float values
    ToolDev& T = ctx->tool;
    T.ncyl = n_cyl;
    double z = 0.0, rho = 0.0, pm = 0.0;
    for (int k = 0; k < n_cyl; ++k) {
        T.z0[k] = (float)z;
        z += tool[k].height;
        T.z1[k] = (float)z;
        T.R[k] = tool[k].radius;
        pm = std::max(pm, (double)tool[k].radius);
        T.Rpm[k] = (float)pm;
        rho = std::max(rho, std::sqrt(z * z + (double)tool[k].radius * tool[k].radius));
    }
    for (int k = 0; k < n_cyl; ++k) {
        float mn = tool[k].radius;
        for (int j = k; j < n_cyl; ++j) mn = std::min(mn, tool[j].radius);
        T.Rin[k] = mn;
    }
    for (int k = n_cyl; k < AM_MAX_CYL; ++k) {  // padding read by the unrolled cheap-cone select
        T.z0[k] = 3.0e38f;
        T.z1[k] = 3.0e38f;
        T.R[k] = T.R[n_cyl - 1];
        T.Rin[k] = T.Rin[n_cyl - 1];
        T.Rpm[k] = T.Rpm[n_cyl - 1];
    }
    for (int k = 0; k < AM_MAX_CYL; ++k)
        for (int set = 0; set < 2; ++set)
            for (int e = 0; e < 2; ++e) {
                const double zc = k < n_cyl ? (double)(e ? T.z1[k] : T.z0[k]) : 1.0;
                const double Rc = k < n_cyl ? (double)(set ? T.Rin[k] : T.R[k]) : 1.0;
                const double dc = std::sqrt(zc * zc + Rc * Rc);
                T.cD[set][e][k] = (float)dc;
                T.ciD[set][e][k] = (float)(1.0 / dc);
            }
    T.R_first = T.Rpm[0];
    T.nbp = 0;
    for (int k = 0; k < AM_MAX_CYL; ++k) {
        T.bp_z[k] = 3.0e38f;
        T.bp_R[k] = T.Rpm[n_cyl - 1];
    }
    for (int k = 1; k < n_cyl; ++k)
        if (T.Rpm[k] > T.Rpm[k - 1]) {
            T.bp_z[T.nbp] = T.z0[k];
            T.bp_R[T.nbp] = T.Rpm[k];
            ++T.nbp;
        }
    T.L = (float)z;
    T.rho_max = (float)rho;
    GridDev& G = ctx->grid;
    G.m = m;
    G.n = n;
    G.W = (n + 31) / 32;
    const double PI = 3.14159265358979323846;
    G.dphi = (float)(PI / m);
    G.inv_dphi = (float)(m / PI);
    G.dgam = (float)(2.0 * PI / n);
    G.inv_dgam = (float)(n / (2.0 * PI));
    G.rowscan = AM_CMAP_ROWSCAN;
    G.brute = AM_CMAP_BRUTE;
    G.cblock = AM_CMAP_BLOCK;
    G.far_cos = AM_CMAP_FAR > 0 ? (float)std::cos(AM_CMAP_FAR * M_PI / 180.0) : -2.f;
    ctx->MW = m * G.W;
    int rc;
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) {
        cudaGetLastError();
        delete ctx;
        return AM_ECUDA;
    }
    ctx->sms = prop.multiProcessorCount;
    std::vector<float> tab(2 * m + 2 * n);
    for (int i = 0; i < m; ++i) {
        const double ph = (i + 0.5) * PI / m;
        tab[i] = (float)std::cos(ph);
        tab[m + i] = (float)std::sin(ph);
    }
    for (int j = 0; j < n; ++j) {
        const double ga = (j + 0.5) * 2.0 * PI / n;
        tab[2 * m + j] = (float)std::cos(ga);
        tab[2 * m + n + j] = (float)std::sin(ga);
    }
    auto bail = [&](int code) {
        am_destroy(ctx);
        return code;
    };
    if (cudaMalloc(&ctx->d_tab, tab.size() * sizeof(float)) != cudaSuccess ||
        cudaMemcpy(ctx->d_tab, tab.data(), tab.size() * sizeof(float), cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMalloc(&ctx->d_ctr, kCtrStride * sizeof(unsigned long long)) != cudaSuccess ||
        cudaMalloc(&ctx->d_am, (size_t)ctx->MW * sizeof(uint32_t)) != cudaSuccess) {
        cudaGetLastError();
        return bail(AM_ENOMEM);
    }
    ctx->am_cap_maps = 1;
    // finer orientation grids (C4, 128 x 128) are faster with a coarser default map (B200 sweep,
    // profiles/r2v_sweep.txt: 12.50 -> 12.28 us per map at T = 80)
    if ((long long)m * n >= 128ll * 128) ctx->cmapT = 80;
    {
        const std::vector<float> tex = make_texels(ctx->cmapT);
        if (cudaMalloc(&ctx->d_texels, tex.size() * sizeof(float)) != cudaSuccess ||
            cudaMemcpy(ctx->d_texels, tex.data(), tex.size() * sizeof(float), cudaMemcpyHostToDevice) != cudaSuccess ||
            cudaMalloc(&ctx->d_cmap, tex.size() / 4 * sizeof(float4)) != cudaSuccess ||
            cudaMalloc(&ctx->d_cmap_ones, tex.size() / 4 * sizeof(float4)) != cudaSuccess) {
            cudaGetLastError();
            return bail(AM_ENOMEM);
        }
    }
    if (set_texels1(ctx, std::min(ctx->cmapT1, ctx->cmapT)) != AM_OK) return bail(AM_ENOMEM);
    {
        const std::vector<float4> ones((size_t)6 * ctx->cmapT * ctx->cmapT, make_float4(1.f, 0.f, 1.f, 0.f));
        if (cudaMemcpy(ctx->d_cmap_ones, ones.data(), ones.size() * sizeof(float4), cudaMemcpyHostToDevice) !=
            cudaSuccess) {
            cudaGetLastError();
            return bail(AM_ECUDA);
        }
    }
    if (cudaMalloc(&ctx->d_recs, (size_t)kRecCap * sizeof(ConeRec)) != cudaSuccess ||
        cudaMalloc(&ctx->d_tasks, (size_t)kTaskCap * sizeof(unsigned long long)) != cudaSuccess) {
        cudaGetLastError();
        return bail(AM_ENOMEM);
    }
    if ((rc = ensure_queue(ctx, 1 << 22)) != AM_OK) return bail(rc);
    if ((rc = configure_launch(ctx)) != AM_OK) return bail(rc);
    *out = ctx;
    return AM_OK;
}

int am_upload_voxels(am_ctx* ctx, const float* centers_xyz, const float* half_sizes, int64_t N,
                     int src_is_device) {
    if (!ctx) return AM_EINVAL;
    ctx->uploaded = false;  // (a failed upload leaves no model: AM_ESTATE until one succeeds)
    if (N < 0) return fail(ctx, AM_EINVAL, "N < 0");
    if (N > 0x7fffffffLL) return fail(ctx, AM_EINVAL, "N exceeds 2^31 - 1");
    if (N > 0 && (!centers_xyz || !half_sizes)) return fail(ctx, AM_EINVAL, "NULL voxel array");
    ++ctx->gen;
    DeviceGuard dg(ctx->device);
    if (!dg.ok) return fail(ctx, AM_ECUDA, "cannot select device %d", ctx->device);
    if (N == 0) {
        ctx->N = 0;
        ctx->uploaded = true;
        ctx->o_built = false;
        return AM_OK;
    }
    const float* dc = centers_xyz;
    const float* dh = half_sizes;
    float* tmp_c = nullptr;
    float* tmp_h = nullptr;
    float4* raw = nullptr;
    unsigned int* bbox = nullptr;
    unsigned long long* bad = nullptr;
    unsigned long long* keys = nullptr;
    unsigned long long* keys2 = nullptr;
    unsigned int* ids = nullptr;
    unsigned int* ids2 = nullptr;
    void* cubtmp = nullptr;
    int rc = AM_OK;
    auto cleanup = [&]() {
        cudaFree(tmp_c);
        cudaFree(tmp_h);
        cudaFree(raw);
        cudaFree(bbox);
        cudaFree(bad);
        cudaFree(keys);
        cudaFree(keys2);
        cudaFree(ids);
        cudaFree(ids2);
        cudaFree(cubtmp);
    };
#define UK(call)                                                                               \
    do {                                                                                       \
        cudaError_t e_ = (call);                                                               \
        if (e_ != cudaSuccess) {                                                               \
            cudaGetLastError();                                                                \
            cleanup();                                                                         \
            return fail(ctx, e_ == cudaErrorMemoryAllocation ? AM_ENOMEM : AM_ECUDA, "%s: %s", #call, \
                        cudaGetErrorString(e_));                                               \
        }                                                                                      \
    } while (0)
    if (!src_is_device) {
        UK(cudaMalloc(&tmp_c, (size_t)N * 3 * sizeof(float)));
        UK(cudaMalloc(&tmp_h, (size_t)N * sizeof(float)));
        UK(cudaMemcpy(tmp_c, centers_xyz, (size_t)N * 3 * sizeof(float), cudaMemcpyHostToDevice));
        UK(cudaMemcpy(tmp_h, half_sizes, (size_t)N * sizeof(float), cudaMemcpyHostToDevice));
        dc = tmp_c;
        dh = tmp_h;
    }
    if (ctx->vox_cap < N) {
        cudaFree(ctx->d_vox);
        cudaFree(ctx->d_live_full);
        ctx->d_vox = nullptr;
        ctx->d_live_full = nullptr;
        ctx->vox_cap = 0;
        UK(cudaMalloc(&ctx->d_vox, (size_t)N * sizeof(float4)));
        UK(cudaMalloc(&ctx->d_live_full, (size_t)N * sizeof(unsigned int)));
        ctx->vox_cap = N;
    }
    {
        // the live list of each batched map slot: live voxels are a small fraction of the model once the
        // coarse levels and the clear-direction map are in (~0.04 % at C3), so it holds max(2^20, N / 8)
        // entries (at most N; AM_OPT_LIVE_CAP), not N -- an overflow is re-streamed (live_overflow_rescan)
        const long long want = ctx->live_cap_opt > 0
                                   ? std::min<long long>(ctx->live_cap_opt, ctx->vox_cap)
                                   : std::min<long long>(ctx->vox_cap, std::max<long long>(1ll << 20, ctx->vox_cap / 8));
        if (want != ctx->live_cap || !ctx->d_live) {
            cudaFree(ctx->d_live);
            ctx->d_live = nullptr;
            ctx->live_cap = 0;
            UK(cudaMalloc(&ctx->d_live, (size_t)ctx->slots * want * sizeof(unsigned int)));
            ctx->live_cap = want;
            ++ctx->gen;
        }
    }
    UK(cudaMalloc(&raw, (size_t)N * sizeof(float4)));
    UK(cudaMalloc(&bbox, 6 * sizeof(unsigned int)));
    UK(cudaMalloc(&bad, sizeof(unsigned long long)));
    const unsigned int init[6] = {0xffffffffu, 0xffffffffu, 0xffffffffu, 0u, 0u, 0u};
    UK(cudaMemcpy(bbox, init, sizeof init, cudaMemcpyHostToDevice));
    UK(cudaMemset(bad, 0, sizeof(unsigned long long)));
    const int blocks = ctx->sms * 8;
    pack_validate_kernel<<<blocks, 256>>>(dc, dh, N, raw, bbox, bad);
    UK(cudaGetLastError());
    unsigned long long nbad = 0;
    UK(cudaMemcpy(&nbad, bad, sizeof nbad, cudaMemcpyDeviceToHost));
    if (nbad) {
        cleanup();
        return fail(ctx, AM_EINVAL, "%llu voxels with a non-finite value or half size <= 0", nbad);
    }
    {
        unsigned int hb[6];
        UK(cudaMemcpy(hb, bbox, sizeof hb, cudaMemcpyDeviceToHost));
        for (int k = 0; k < 6; ++k) {  // ordered-int encoding back to float (see float_to_ordered)
            const unsigned int u = (hb[k] & 0x80000000u) ? (hb[k] & 0x7fffffffu) : ~hb[k];
            float f;
            std::memcpy(&f, &u, sizeof f);
            ctx->bbox[k] = f;
        }
    }
    if (ctx->morton) {
        UK(cudaMalloc(&keys, (size_t)N * sizeof(unsigned long long)));
        UK(cudaMalloc(&keys2, (size_t)N * sizeof(unsigned long long)));
        UK(cudaMalloc(&ids, (size_t)N * sizeof(unsigned int)));
        UK(cudaMalloc(&ids2, (size_t)N * sizeof(unsigned int)));
        morton_keys_kernel<<<blocks, 256>>>(raw, N, bbox, keys, ids);
        UK(cudaGetLastError());
        size_t tb = 0;
        UK(cub::DeviceRadixSort::SortPairs(nullptr, tb, keys, keys2, ids, ids2, (int)N, 0, 63));
        UK(cudaMalloc(&cubtmp, tb));
        UK(cub::DeviceRadixSort::SortPairs(cubtmp, tb, keys, keys2, ids, ids2, (int)N, 0, 63));
        gather_kernel<<<blocks, 256>>>(raw, ids2, N, ctx->d_vox);
        UK(cudaGetLastError());
    } else {
        UK(cudaMemcpy(ctx->d_vox, raw, (size_t)N * sizeof(float4), cudaMemcpyDeviceToDevice));
    }
    // bricks of kThreads consecutive (Morton-ordered) voxels and their bounding spheres
    cudaFree(ctx->d_bricks);
    cudaFree(ctx->d_brick_list);
    ctx->d_bricks = nullptr;
    ctx->d_brick_list = nullptr;
    ctx->nbricks = (unsigned int)((N + kThreads - 1) / kThreads);
    UK(cudaMalloc(&ctx->d_bricks, (size_t)ctx->nbricks * sizeof(float4)));
    UK(cudaMalloc(&ctx->d_brick_list, (size_t)ctx->slots * blist_words(ctx) * sizeof(unsigned int)));
    brick_bounds_kernel<<<(unsigned)(((long long)ctx->nbricks * 32 + 255) / 256), 256>>>(ctx->d_vox, N, ctx->d_bricks,
                                                                                        ctx->nbricks, kThreads);
    UK(cudaGetLastError());
    cudaFree(ctx->d_subs);
    cudaFree(ctx->d_supers);
    ctx->d_subs = ctx->d_supers = nullptr;
    {
        const unsigned int nsup = (ctx->nbricks + 7) / 8;
        if (nsup > 0) {
            UK(cudaMalloc(&ctx->d_supers, (size_t)nsup * sizeof(float4)));
            brick_bounds_kernel<<<(unsigned)(((long long)nsup * 32 + 255) / 256), 256>>>(ctx->d_vox, N, ctx->d_supers,
                                                                                         nsup, 8 * kThreads);
            UK(cudaGetLastError());
        }
        const unsigned int nsub = (unsigned int)((N + 31) / 32);
        if (nsub > 0) {
            UK(cudaMalloc(&ctx->d_subs, (size_t)nsub * sizeof(float4)));
            brick_bounds_kernel<<<(unsigned)(((long long)nsub * 32 + 255) / 256), 256>>>(ctx->d_vox, N, ctx->d_subs,
                                                                                         nsub, 32);
            UK(cudaGetLastError());
        }
    }
    // coarse levels for the clear-direction map: level 0 = the n0 largest
    // voxels, level 1 = the next ones up to n1 plus every 512th voxel
    cudaFree(ctx->d_coarse);
    cudaFree(ctx->d_l1subs);
    ctx->d_coarse = ctx->d_l1subs = nullptr;
    ctx->n_l0 = ctx->n_l1 = 0;
    if (N >= 2048) {
        const long long n0 = std::min<long long>(N, std::max<long long>(1024, N / AM_L0_DIV));
        const long long n1 = std::min<long long>(N, std::max<long long>(8192, N / AM_L1_DIV));
        // strided sample: every AM_L1_STRIDE-th voxel, at least AM_L1_MIN_SAMPLE voxels (small models)
        long long stride = AM_L1_STRIDE;
        if (N / stride < AM_L1_MIN_SAMPLE) stride = std::max<long long>(1, N / AM_L1_MIN_SAMPLE);
        if (ctx->l1_sample > 0) stride = std::max<long long>(1, N / ctx->l1_sample);  // AM_OPT_L1_SAMPLE
        const long long ns = std::min<long long>(N / stride, N - n1);  // level 1 fits the live lists (N)
        unsigned int *sk = nullptr, *sk2 = nullptr, *si = nullptr, *si2 = nullptr, *cid = nullptr;
        void* ct = nullptr;
        auto cfree = [&]() {
            cudaFree(sk); cudaFree(sk2); cudaFree(si); cudaFree(si2); cudaFree(cid); cudaFree(ct);
        };
#define CUK(call)                                                                              \
        do {                                                                                   \
            cudaError_t e_ = (call);                                                           \
            if (e_ != cudaSuccess) {                                                           \
                cudaGetLastError();                                                            \
                cfree();                                                                       \
                cleanup();                                                                     \
                return fail(ctx, e_ == cudaErrorMemoryAllocation ? AM_ENOMEM : AM_ECUDA, "%s: %s", #call, \
                            cudaGetErrorString(e_));                                           \
            }                                                                                  \
        } while (0)
        CUK(cudaMalloc(&sk, (size_t)N * 4));
        CUK(cudaMalloc(&sk2, (size_t)N * 4));
        CUK(cudaMalloc(&si, (size_t)N * 4));
        CUK(cudaMalloc(&si2, (size_t)N * 4));
        CUK(cudaMalloc(&cid, (size_t)(n1 + ns) * 4));
        size_keys_kernel<<<blocks, 256>>>(ctx->d_vox, N, sk, si);
        CUK(cudaGetLastError());
        size_t tb = 0;
        CUK(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, sk, sk2, si, si2, (int)N, 0, 32));
        CUK(cudaMalloc(&ct, tb));
        CUK(cub::DeviceRadixSort::SortPairsDescending(ct, tb, sk, sk2, si, si2, (int)N, 0, 32));
        CUK(cudaMemcpy(cid, si2, (size_t)n1 * 4, cudaMemcpyDeviceToDevice));
        if (ns > 0) {
            strided_ids_kernel<<<blocks, 256>>>(cid + n1, ns, stride);
            CUK(cudaGetLastError());
        }
        // level 1 (after the n0 largest) in model (Morton) order, so that every 32 consecutive level-1
        // voxels are a compact group with a useful bounding sphere (the batched level-1 cone launch
        // skips a group whose sphere cannot reach a clear cell of the map after level 0)
        if (n1 + ns > n0) {
            size_t tb1 = 0;
            const int nl1 = (int)(n1 + ns - n0);
            CUK(cub::DeviceRadixSort::SortKeys(nullptr, tb1, cid + n0, sk, nl1, 0, 32));
            if (tb1 > tb) {
                cudaFree(ct);
                ct = nullptr;
                CUK(cudaMalloc(&ct, tb1));
                tb = tb1;
            }
            CUK(cub::DeviceRadixSort::SortKeys(ct, tb, cid + n0, sk, nl1, 0, 32));
            CUK(cudaMemcpy(cid + n0, sk, (size_t)nl1 * 4, cudaMemcpyDeviceToDevice));
        }
        CUK(cudaMalloc(&ctx->d_coarse, (size_t)(n1 + ns) * sizeof(float4)));
        gather_kernel<<<blocks, 256>>>(ctx->d_vox, cid, n1 + ns, ctx->d_coarse);
        CUK(cudaGetLastError());
        if (n1 + ns > n0) {
            const long long nl1 = n1 + ns - n0;
            const unsigned int ng = (unsigned int)((nl1 + 31) / 32);
            CUK(cudaMalloc(&ctx->d_l1subs, (size_t)ng * sizeof(float4)));
            brick_bounds_kernel<<<(unsigned)(((long long)ng * 32 + 255) / 256), 256>>>(ctx->d_coarse + n0, nl1,
                                                                                       ctx->d_l1subs, ng, 32);
            CUK(cudaGetLastError());
        }
        CUK(cudaDeviceSynchronize());
#undef CUK
        cfree();
        ctx->n_l0 = n0;
        ctx->n_l1 = n1 + ns;
    }
    if (ctx->d_wit)  // (AM_OPT_REUSE witnesses name voxels of the previous model)
        UK(cudaMemset(ctx->d_wit, 0xff, (size_t)ctx->contrib_slots * 2 * ctx->grid.m * ctx->grid.n * sizeof(unsigned int)));
    UK(cudaDeviceSynchronize());
#undef UK
    cleanup();
    ctx->N = N;
    ctx->uploaded = true;
    ctx->o_built = false;  // the octree belongs to the previous model
    return rc;
}

int am_compute(am_ctx* ctx, const float pivot[3], uint32_t* am_out, int dst_is_device,
               void* cuda_stream, am_stats* stats) {
    if (!ctx) return AM_EINVAL;
    int rc = check_pivot(ctx, pivot);
    if (rc) return rc;
    if (!am_out) return fail(ctx, AM_EINVAL, "am_out is NULL");
    if (!ctx->uploaded) return fail(ctx, AM_ESTATE, "am_compute before am_upload_voxels");
    DeviceGuard dg(ctx->device);
    if (!dg.ok) return fail(ctx, AM_ECUDA, "cannot select device %d", ctx->device);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    if ((rc = stream_begin(ctx, s)) != AM_OK) return rc;
    uint32_t* gam = dst_is_device ? am_out : ctx->d_am;
    if ((ctx->diag & 32) && fused_ok(ctx)) {  // (diagnostics: one pivot through the batched phase launches)
        if ((rc = launch_batch_layers(ctx, pivot, 1, gam, s)) != AM_OK) return rc;
    } else if ((rc = launch_aica(ctx, pivot, gam, s)) != AM_OK) {
        return rc;
    }
    if (!dst_is_device)
        CK(cudaMemcpyAsync(am_out, gam, (size_t)ctx->MW * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    if ((rc = stream_end(ctx, s)) != AM_OK) return rc;
    if (stats) {
        unsigned long long h[kCtrWords];
        CK(cudaMemcpyAsync(h, ctx->d_ctr, sizeof h, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        int64_t* o = reinterpret_cast<int64_t*>(stats);
        static_assert(sizeof(am_stats) == (ST_PASSED + 3) * sizeof(int64_t), "am_stats mirrors StatIdx");
        for (int k = 0; k < ST_PASSED; ++k) o[k] = (int64_t)h[1 + k];
        stats->rows_skipped_full = (int64_t)h[1 + ST_ROWFULL];
        // every voxel goes through the filter once; the rest of it was dropped
        o[ST_SKIPPED] = (int64_t)ctx->N - (int64_t)h[1 + ST_CULLED] - (int64_t)h[1 + ST_PASSED];
        // (fused path: kept bricks in the high word, kept sub-bricks -- the list length -- in the low word)
        stats->bricks_kept = (ctx->bricks_on && ctx->d_bricks && !(fused_ok(ctx) && small_model(ctx)))
                                 ? (int64_t)(fused_ok(ctx) ? (h[kCtrBricks] >> 32) : (h[kCtrBricks] & 0xffffffffull))
                                 : (int64_t)ctx->nbricks;  // (small models: every brick is read)
        stats->level_voxels = ctx->phases == 0 ? 0 : ctx->phases == 1 ? ctx->n_l0 : ctx->n_l1;
        if ((rc = print_phase_times(ctx)) != AM_OK) return rc;
    } else if (!dst_is_device) {
        CK(cudaStreamSynchronize(s));
    }
    return AM_OK;
}

int am_compute_batch(am_ctx* ctx, const float* pivots, int64_t P, uint32_t* am_out, int dst_is_device,
                     void* cuda_stream) {
    if (!ctx) return AM_EINVAL;
    if (P < 0) return fail(ctx, AM_EINVAL, "P < 0");
    if (P > 0 && (!pivots || !am_out)) return fail(ctx, AM_EINVAL, "NULL pivots or am_out");
    for (int64_t k = 0; k < 3 * P; ++k)
        if (!is_finite_f(pivots[k])) return fail(ctx, AM_EINVAL, "pivot %lld is not finite", (long long)(k / 3));
    if (!ctx->uploaded) return fail(ctx, AM_ESTATE, "am_compute_batch before am_upload_voxels");
    if (P == 0) return AM_OK;
    DeviceGuard dg(ctx->device);
    if (!dg.ok) return fail(ctx, AM_ECUDA, "cannot select device %d", ctx->device);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    int rc;
    if ((rc = stream_begin(ctx, s)) != AM_OK) return rc;
    uint32_t* dst = am_out;
    if (!dst_is_device) {
        if (ctx->am_cap_maps < P) {
            cudaFree(ctx->d_am);
            ctx->d_am = nullptr;
            ctx->am_cap_maps = 0;
            CK(cudaMalloc(&ctx->d_am, (size_t)P * ctx->MW * sizeof(uint32_t)));
            ctx->am_cap_maps = P;
        }
        dst = ctx->d_am;
    }
    const int K = (int)std::min<int64_t>(P, ctx->batch);
    if (K > 1 && fused_ok(ctx) && (ctx->diag & 8)) {
        // diagnostic: one cooperative launch, K CTA groups taking pivots from a queue
        const int Kg = std::min(K, (int)kMaxSlots);
        if ((rc = ensure_slots(ctx, Kg)) != AM_OK) return rc;
        if ((rc = launch_fused_batch(ctx, pivots, P, Kg, dst, s)) != AM_OK) return rc;
    } else if (K > 1 && fused_ok(ctx)) {
        // the batch phase by phase, up to ctx->batch pivots per launch (8(f) NEXT 2)
        if ((rc = launch_batch_layers(ctx, pivots, P, dst, s)) != AM_OK) return rc;
    } else {
        for (int64_t k = 0; k < P; ++k)
            if ((rc = launch_aica(ctx, pivots + 3 * k, dst + k * ctx->MW, s)) != AM_OK) return rc;
    }
    if (!dst_is_device) CK(cudaMemcpyAsync(am_out, dst, (size_t)P * ctx->MW * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    if ((rc = stream_end(ctx, s)) != AM_OK) return rc;
    if (!dst_is_device) CK(cudaStreamSynchronize(s));
    if (ctx->diag_ts) {
        CK(cudaStreamSynchronize(s));
        if ((rc = print_phase_times(ctx)) != AM_OK) return rc;
    }
    return AM_OK;
}

int am_compute_baseline(am_ctx* ctx, const float pivot[3], uint32_t* am_out, int dst_is_device,
                        void* cuda_stream) {
    if (!ctx) return AM_EINVAL;
    int rc = check_pivot(ctx, pivot);
    if (rc) return rc;
    if (!am_out) return fail(ctx, AM_EINVAL, "am_out is NULL");
    if (!ctx->uploaded) return fail(ctx, AM_ESTATE, "am_compute_baseline before am_upload_voxels");
    DeviceGuard dg(ctx->device);
    if (!dg.ok) return fail(ctx, AM_ECUDA, "cannot select device %d", ctx->device);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    if ((rc = stream_begin(ctx, s)) != AM_OK) return rc;
    uint32_t* gam = dst_is_device ? am_out : ctx->d_am;
    CK(cudaMemsetAsync(gam, 0, (size_t)ctx->MW * sizeof(uint32_t), s));
    if (ctx->N > 0) {
        StreamParams p = make_params(ctx, pivot, gam);
        const int ncell = ctx->grid.m * ctx->grid.n;
        int g = ctx->sms * 8;
        if (g > ncell) g = ncell;
        int rc;
        if ((rc = kchain(ctx, s))) return rc;
        baseline_kernel<<<g, kThreads, 0, s>>>(p, ctx->baseline_reject);
        if ((rc = kmark(ctx, s, AM_K_BASELINE))) return rc;
    }
    if (!dst_is_device) CK(cudaMemcpyAsync(am_out, gam, (size_t)ctx->MW * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    if ((rc = stream_end(ctx, s)) != AM_OK) return rc;
    if (!dst_is_device) CK(cudaStreamSynchronize(s));
    return AM_OK;
}

int am_set_option(am_ctx* ctx, int key, int64_t value) {
    if (!ctx) return AM_EINVAL;
    DeviceGuard dg(ctx->device);
    // options that shape the batched launch chain invalidate its captured graph; timing, the
    // baseline's reject, the upload-time options and the graph switch itself do not
    if (key != AM_OPT_KERNEL_TIMING && key != AM_OPT_BASELINE_REJECT && key != AM_OPT_MORTON_SORT &&
        key != AM_OPT_L1_SAMPLE && key != AM_OPT_GRAPH)
        ++ctx->gen;
    switch (key) {
    case AM_OPT_GRID_CTAS:
        if (value < 0 || value > (1 << 20)) return fail(ctx, AM_EINVAL, "grid_ctas out of range");
        ctx->grid_ctas = (int)value;
        return AM_OK;
    case AM_OPT_REFRESH_TILES:
        if (value < 1 || value > (1 << 20)) return fail(ctx, AM_EINVAL, "refresh_tiles out of range");
        ctx->refresh_tiles = (int)value;
        return AM_OK;
    case AM_OPT_MORTON_SORT:
        if (value != 0 && value != 1) return fail(ctx, AM_EINVAL, "morton_sort must be 0 or 1");
        ctx->morton = (int)value;
        return AM_OK;
    case AM_OPT_BASELINE_REJECT:
        if (value != 0 && value != 1) return fail(ctx, AM_EINVAL, "baseline_reject must be 0 or 1");
        ctx->baseline_reject = (int)value;
        return AM_OK;
    case AM_OPT_BAND_QUEUE:
        if (value < 1 || value > (1LL << 28)) return fail(ctx, AM_EINVAL, "band queue out of range");
        return ensure_queue(ctx, value);
    case AM_OPT_KERNEL_TIMING:
        if (value < 0 || value > 2) return fail(ctx, AM_EINVAL, "kernel_timing must be 0, 1 or 2");
        ctx->timing = (int)value;
        return AM_OK;
    case AM_OPT_PHASES:
        if (value < 0 || value > 2) return fail(ctx, AM_EINVAL, "phases must be 0, 1 or 2");
        ctx->phases = (int)value;
        return AM_OK;
    case AM_OPT_DIAG:
        if (value < 0 || value > 63) return fail(ctx, AM_EINVAL, "diag must be in [0, 63]");
        if ((value & 3) && !ctx->d_prev) {
            CK(cudaMalloc(&ctx->d_prev, (size_t)ctx->MW * sizeof(uint32_t)));
            CK(cudaMemset(ctx->d_prev, 0, (size_t)ctx->MW * sizeof(uint32_t)));
        }
        if ((value & 4) && !ctx->d_ts) {
            CK(cudaMalloc(&ctx->d_ts, (16 + 4 * kDiagCtas) * sizeof(unsigned long long)));
            CK(cudaMemset(ctx->d_ts, 0, (16 + 4 * kDiagCtas) * sizeof(unsigned long long)));
        }
        ctx->diag = (int)value;
        ctx->diag_ts = (value & 4) != 0;
        return AM_OK;
    case AM_OPT_BRICKS:
        if (value != 0 && value != 1) return fail(ctx, AM_EINVAL, "bricks must be 0 or 1");
        ctx->bricks_on = (int)value;
        return AM_OK;
    case AM_OPT_FUSED:
        if (value != 0 && value != 1) return fail(ctx, AM_EINVAL, "fused must be 0 or 1");
        ctx->fused = (int)value;
        return AM_OK;
    case AM_OPT_BATCH:
        if (value < 1 || value > kMaxBatch) return fail(ctx, AM_EINVAL, "batch must be in [1, %d]", kMaxBatch);
        ctx->batch = (int)value;
        return AM_OK;
    case AM_OPT_BAND_SUBDIV:
        if (value < 0 || value > 3) return fail(ctx, AM_EINVAL, "band_subdiv must be in [0, 3]");
        ctx->band_vdepth = (int)value;
        return AM_OK;
    case AM_OPT_CMAP_ROWSCAN:
        if (value < 0 || value > (1 << 21)) return fail(ctx, AM_EINVAL, "cmap_rowscan must be in [0, 2^21]");
        ctx->grid.rowscan = (int)value;
        return AM_OK;
    case AM_OPT_CMAP_BRUTE:
        if (value < 0 || value > (1 << 21)) return fail(ctx, AM_EINVAL, "cmap_brute must be in [0, 2^21]");
        ctx->grid.brute = (int)value;
        return AM_OK;
    case AM_OPT_CMAP_BLOCK:
        if (value != 4 && value != 8) return fail(ctx, AM_EINVAL, "cmap_block must be 4 or 8");
        ctx->grid.cblock = (int)value;
        return AM_OK;
    case AM_OPT_CMAP_FAR:
        if (value < 0 || value > 180) return fail(ctx, AM_EINVAL, "cmap_far must be in [0, 180] degrees");
        ctx->grid.far_cos = value > 0 ? (float)std::cos((double)value * M_PI / 180.0) : -2.f;
        return AM_OK;
    case AM_OPT_MAP_CTAS:
        if (value < 0 || value > 4096) return fail(ctx, AM_EINVAL, "map_ctas must be in [0, 4096]");
        ctx->bk_map_ctas = (int)value;
        return AM_OK;
    case AM_OPT_SUBBRICKS:
        if (value < 0 || value > 3) return fail(ctx, AM_EINVAL, "subbricks must be in [0, 3]");
        ctx->subs_on = (int)value;
        return AM_OK;
    case AM_OPT_GRAPH:
        if (value != 0 && value != 1) return fail(ctx, AM_EINVAL, "graph must be 0 or 1");
        ctx->use_graph = (int)value;
        return AM_OK;
    case AM_OPT_BATCH_LANES:
        if (value < 1 || value > kMaxLanes) return fail(ctx, AM_EINVAL, "batch_lanes must be in [1, %d]", kMaxLanes);
        ctx->lanes = (int)value;
        return AM_OK;
    case AM_OPT_REUSE:
        if (value != 0 && value != 1) return fail(ctx, AM_EINVAL, "reuse must be 0 or 1");
        ctx->reuse = (int)value;
        return AM_OK;
    case AM_OPT_STAGE_FUSION:
        if (value < 0 || value > 7) return fail(ctx, AM_EINVAL, "stage_fusion must be in [0, 7]");
        ctx->stage_fusion = (int)value;
        return AM_OK;
    case AM_OPT_L1_SUBS:
        if (value != 0 && value != 1) return fail(ctx, AM_EINVAL, "l1_subs must be 0 or 1");
        ctx->l1_subs = (int)value;
        return AM_OK;
    case AM_OPT_L1_SPARSE:
        if (value < 0 || value > (1 << 20)) return fail(ctx, AM_EINVAL, "l1_sparse must be in [0, 2^20]");
        ctx->l1_sparse = (int)value;
        return AM_OK;
    case AM_OPT_LIVE_CAP:
        if (value < 0 || value > INT32_MAX) return fail(ctx, AM_EINVAL, "live_cap must be in [0, 2^31-1]");
        ctx->live_cap_opt = value;  // taken at the next am_upload_voxels
        return AM_OK;
    case AM_OPT_PDL:
        if (value != 0 && value != 1) return fail(ctx, AM_EINVAL, "pdl must be 0 or 1");
        ctx->pdl = (int)value;
        return AM_OK;
    case AM_OPT_STREAM_TMA:
        if (value < 0 || value > kTmaShapes) return fail(ctx, AM_EINVAL, "stream_tma must be in [0, %d]", kTmaShapes);
        ctx->stream_tma = (int)value;
        return AM_OK;
    case AM_OPT_L1_SAMPLE:
        if (value < 0 || value > INT32_MAX) return fail(ctx, AM_EINVAL, "l1_sample must be in [0, 2^31-1]");
        ctx->l1_sample = value;  // taken at the next am_upload_voxels
        return AM_OK;
    case AM_OPT_CMAP_T1:
        if (value < 4 || value > ctx->cmapT) return fail(ctx, AM_EINVAL, "cmap_T1 must be in [4, cmap_T]");
        return set_texels1(ctx, (int)value);
    case AM_OPT_CMAP_T:
        if (value < 4 || value > 256) return fail(ctx, AM_EINVAL, "cmap_T must be in [4, 256]");
        return set_cmap_T(ctx, (int)value);
    default:
        return fail(ctx, AM_EINVAL, "unknown option %d", key);
    }
}

int am_kernel_time(am_ctx* ctx, double* total_ms, int64_t* launches) {
    if (!ctx) return AM_EINVAL;
    if (!total_ms || !launches) return fail(ctx, AM_EINVAL, "NULL output");
    DeviceGuard dg(ctx->device);
    double tot = 0.0;
    for (size_t k = 0; k < ctx->ev_used; ++k) {
        float ms = 0.f;
        CK(cudaEventSynchronize(ctx->ev_stop[k]));
        CK(cudaEventElapsedTime(&ms, ctx->ev_start[k], ctx->ev_stop[k]));
        tot += ms;
    }
    *total_ms = tot;
    *launches = (int64_t)ctx->ev_used;
    ctx->ev_used = 0;
    return AM_OK;
}

int am_kernel_stats(am_ctx* ctx, double* ms, int64_t* launches) {
    if (!ctx) return AM_EINVAL;
    if (!ms || !launches) return fail(ctx, AM_EINVAL, "NULL output");
    DeviceGuard dg(ctx->device);
    for (int k = 0; k < AM_K_COUNT; ++k) {
        ms[k] = 0.0;
        launches[k] = (int64_t)ctx->k_launches[k];
        ctx->k_launches[k] = 0;
    }
    for (size_t j = 0; j < ctx->kmarks.size(); ++j) {
        float t = 0.f;
        CK(cudaEventSynchronize(ctx->kev[ctx->kmarks[j].second]));
        CK(cudaEventElapsedTime(&t, ctx->kev[ctx->kmark_begin[j]], ctx->kev[ctx->kmarks[j].second]));
        ms[ctx->kmarks[j].first] += t;
    }
    ctx->kmarks.clear();
    ctx->kmark_begin.clear();
    ctx->kev_used = 0;
    ctx->kev_prev = -1;
    return AM_OK;
}

const char* am_kernel_name(int k) {
    static const char* names[AM_K_COUNT] = {
        "l0_cones", "l0_rows", "clear_map", "l1_cones", "l1_rows", "bricks", "voxels",
        "live_cones", "live_rows", "band", "fused_pipeline", "filter", "baseline", "layout",
        "ica_memo", "octree", "init", "level0", "level1", "stream"};
    return (k >= 0 && k < AM_K_COUNT) ? names[k] : nullptr;
}

// ---------------------------------------------------------------------------
// Octree of the resident model for the paper's orientation-per-thread schemes
// (octree.cuh).  Host-side build: every leaf's level and cell in the declared
// root frame, a sort by the Morton code of its first finest-level cell, then
// the nodes level by level (BFS), children of a node contiguous.
// ---------------------------------------------------------------------------
namespace {

uint64_t spread3(uint64_t x) {  // 21 bits -> every third bit
    x &= 0x1fffffull;
    x = (x | x << 32) & 0x1f00000000ffffull;
    x = (x | x << 16) & 0x1f0000ff0000ffull;
    x = (x | x << 8) & 0x100f00f00f00f00full;
    x = (x | x << 4) & 0x10c30c30c30c30c3ull;
    x = (x | x << 2) & 0x1249249249249249ull;
    return x;
}

}  // namespace

int am_build_octree(am_ctx* ctx, const float root_lo[3], float root_size, int64_t* n_nodes) {
    if (!ctx) return AM_EINVAL;
    if (!root_lo || !(root_size > 0.f) || !is_finite_f(root_size)) return fail(ctx, AM_EINVAL, "bad root cube");
    for (int k = 0; k < 3; ++k)
        if (!is_finite_f(root_lo[k])) return fail(ctx, AM_EINVAL, "root_lo[%d] is not finite", k);
    if (!ctx->uploaded) return fail(ctx, AM_ESTATE, "am_build_octree before am_upload_voxels");
    DeviceGuard dg(ctx->device);
    if (!dg.ok) return fail(ctx, AM_ECUDA, "cannot select device %d", ctx->device);
    const long long N = ctx->N;
    std::vector<float4> leaf((size_t)N);
    if (N > 0) CK(cudaMemcpy(leaf.data(), ctx->d_vox, (size_t)N * sizeof(float4), cudaMemcpyDeviceToHost));
    // level and cell of every leaf
    std::vector<int> lev((size_t)N);
    std::vector<uint32_t> cx((size_t)N * 3);
    int Lmax = 0;
    for (long long i = 0; i < N; ++i) {
        const double s = (double)root_size / (2.0 * leaf[i].w);
        const int l = (int)std::lround(std::log2(s));
        if (l < 0 || l > 20 || std::fabs(s - std::ldexp(1.0, l)) > 1e-3 * std::ldexp(1.0, l))
            return fail(ctx, AM_EINVAL, "voxel %lld: half size %g is not root_size / 2^(l+1)", i, leaf[i].w);
        lev[i] = l;
        Lmax = std::max(Lmax, l);
        const double cell = (double)root_size / std::ldexp(1.0, l);
        const float c3[3] = {leaf[i].x, leaf[i].y, leaf[i].z};
        for (int a = 0; a < 3; ++a) {
            const double f = (c3[a] - (double)root_lo[a]) / cell - 0.5;
            const long long q = std::llround(f);
            if (q < 0 || q >= (1ll << l) || std::fabs(f - (double)q) > 1e-2)
                return fail(ctx, AM_EINVAL, "voxel %lld is not a cell of the root cube's level %d", i, l);
            cx[3 * i + a] = (uint32_t)q;
        }
    }
    // sort by the Morton code of each leaf's first finest-level cell
    std::vector<uint64_t> key((size_t)N);
    for (long long i = 0; i < N; ++i) {
        const int sh = Lmax - lev[i];
        key[i] = spread3((uint64_t)cx[3 * i] << sh) | spread3((uint64_t)cx[3 * i + 1] << sh) << 1 |
                 spread3((uint64_t)cx[3 * i + 2] << sh) << 2;
    }
    std::vector<long long> ord((size_t)N);
    for (long long i = 0; i < N; ++i) ord[i] = i;
    std::sort(ord.begin(), ord.end(), [&](long long a, long long b) { return key[a] < key[b]; });
    for (long long t = 0; t + 1 < N; ++t) {  // leaves are disjoint cells
        const long long a = ord[t], b = ord[t + 1];
        const uint64_t span = 1ull << (3 * (Lmax - lev[a]));
        if (key[b] < key[a] + span) return fail(ctx, AM_EINVAL, "voxels %lld and %lld overlap", a, b);
    }
    std::vector<uint64_t> skey((size_t)N);
    for (long long t = 0; t < N; ++t) skey[t] = key[ord[t]];
    // BFS: node = (level, first finest code, leaf range [a, b))
    struct Pend { int L; uint64_t base; long long a, b; };
    std::vector<Pend> q;
    std::vector<float4> box;
    std::vector<int2> link;
    std::vector<long long> level_end;
    if (N > 0) q.push_back({0, 0ull, 0, N});
    size_t head = 0;
    while (head < q.size()) {
        const Pend nd = q[head];
        const size_t self = head++;
        (void)self;
        while ((int)level_end.size() <= nd.L) level_end.push_back(0);
        level_end[nd.L] = (long long)head;
        const long long first = ord[nd.a];
        if (nd.b - nd.a == 1 && lev[first] == nd.L) {  // a leaf: the uploaded voxel itself
            box.push_back(leaf[first]);
            link.push_back(make_int2(0, 0));
            continue;
        }
        for (long long t = nd.a; t < nd.b; ++t)
            if (lev[ord[t]] <= nd.L) return fail(ctx, AM_EINVAL, "voxel %lld overlaps a finer voxel", ord[t]);
        if (nd.L >= Lmax) return fail(ctx, AM_EINVAL, "octree build: inconsistent levels");
        const double cell = (double)root_size / std::ldexp(1.0, nd.L);
        // the node cube from its first finest cell
        uint32_t c3[3] = {0, 0, 0};
        for (int bit = 0; bit < 21; ++bit)
            for (int a = 0; a < 3; ++a) c3[a] |= (uint32_t)((nd.base >> (3 * bit + a)) & 1ull) << bit;
        float4 bx;
        bx.x = (float)(root_lo[0] + ((c3[0] >> (Lmax - nd.L)) + 0.5) * cell);
        bx.y = (float)(root_lo[1] + ((c3[1] >> (Lmax - nd.L)) + 0.5) * cell);
        bx.z = (float)(root_lo[2] + ((c3[2] >> (Lmax - nd.L)) + 0.5) * cell);
        bx.w = (float)(0.5 * cell);
        box.push_back(bx);
        const int firstc = (int)q.size();
        int nc = 0;
        const uint64_t span = 1ull << (3 * (Lmax - nd.L - 1));
        long long a = nd.a;
        for (int c = 0; c < 8 && a < nd.b; ++c) {
            const uint64_t hi = nd.base + (uint64_t)(c + 1) * span;
            const long long b = std::lower_bound(skey.begin() + a, skey.begin() + nd.b, hi) - skey.begin();
            if (b > a) {
                q.push_back({nd.L + 1, nd.base + (uint64_t)c * span, a, b});
                ++nc;
            }
            a = b;
        }
        if ((long long)q.size() > (1ll << 31) - 8) return fail(ctx, AM_ENOMEM, "octree too large");
        link.push_back(make_int2(firstc, nc));
    }
    for (size_t L = 1; L < level_end.size(); ++L) level_end[L] = std::max(level_end[L], level_end[L - 1]);
    cudaFree(ctx->d_onode);
    cudaFree(ctx->d_olink);
    cudaFree(ctx->d_omemo);
    ctx->d_onode = nullptr;
    ctx->d_olink = nullptr;
    ctx->d_omemo = nullptr;
    ctx->o_n = (long long)box.size();
    ctx->o_level_end = level_end;
    if (ctx->o_n > 0) {
        CK(cudaMalloc(&ctx->d_onode, box.size() * sizeof(float4)));
        CK(cudaMalloc(&ctx->d_olink, link.size() * sizeof(int2)));
        CK(cudaMalloc(&ctx->d_omemo, box.size() * sizeof(float4)));
        CK(cudaMemcpy(ctx->d_onode, box.data(), box.size() * sizeof(float4), cudaMemcpyHostToDevice));
        CK(cudaMemcpy(ctx->d_olink, link.data(), link.size() * sizeof(int2), cudaMemcpyHostToDevice));
    }
    if (!ctx->d_ostats) CK(cudaMalloc(&ctx->d_ostats, 4 * sizeof(unsigned long long)));
    ctx->o_built = true;
    if (n_nodes) *n_nodes = ctx->o_n;
    return AM_OK;
}

int am_compute_octree(am_ctx* ctx, const float pivot[3], int scheme, int S, int vdepth, uint32_t* am_out,
                      int dst_is_device, void* cuda_stream, int64_t* stats) {
    if (!ctx) return AM_EINVAL;
    int rc = check_pivot(ctx, pivot);
    if (rc) return rc;
    if (!am_out) return fail(ctx, AM_EINVAL, "am_out is NULL");
    if (scheme < AM_SCHEME_PBOX || scheme > AM_SCHEME_AICA) return fail(ctx, AM_EINVAL, "unknown scheme %d", scheme);
    if (S < 0 || S > 64) return fail(ctx, AM_EINVAL, "S must be in [0, 64]");
    if (vdepth < 0 || vdepth > 3) return fail(ctx, AM_EINVAL, "vdepth must be in [0, 3]");
    if (!ctx->uploaded) return fail(ctx, AM_ESTATE, "am_compute_octree before am_upload_voxels");
    if (!ctx->o_built) return fail(ctx, AM_ESTATE, "am_compute_octree before am_build_octree");
    DeviceGuard dg(ctx->device);
    if (!dg.ok) return fail(ctx, AM_ECUDA, "cannot select device %d", ctx->device);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    if ((rc = stream_begin(ctx, s)) != AM_OK) return rc;
    uint32_t* gam = dst_is_device ? am_out : ctx->d_am;
    CK(cudaMemsetAsync(gam, 0, (size_t)ctx->MW * sizeof(uint32_t), s));
    CK(cudaMemsetAsync(ctx->d_ostats, 0, 4 * sizeof(unsigned long long), s));
    if (ctx->o_n > 0) {
        if ((rc = kchain(ctx, s))) return rc;
        OctParams P{};
        P.box = ctx->d_onode;
        P.link = ctx->d_olink;
        P.memo = ctx->d_omemo;
        P.nmemo = 0;
        P.px = pivot[0];
        P.py = pivot[1];
        P.pz = pivot[2];
        P.tool = ctx->tool;
        P.grid = ctx->grid;
        P.tab = ctx->d_tab;
        P.gam = gam;
        P.vdepth = vdepth;
        P.stats = ctx->d_ostats;
        if ((scheme == AM_SCHEME_MICA || scheme == AM_SCHEME_AICA) && S > 0) {
            // the parallel ICA calculation of the top S levels (levels 0 .. S-1)
            const int L = std::min<int>(S, (int)ctx->o_level_end.size()) - 1;
            P.nmemo = ctx->o_level_end[L];
            const unsigned g = (unsigned)std::max<long long>(1, std::min<long long>((P.nmemo + 255) / 256, ctx->sms * 8));
            ica_memo_kernel<<<g, 256, 0, s>>>(ctx->d_onode, P.nmemo, P.px, P.py, P.pz, ctx->tool, ctx->d_omemo);
            if ((rc = kmark(ctx, s, AM_K_ICA_MEMO))) return rc;
        }
        const unsigned ncell = (unsigned)(ctx->grid.m * ctx->grid.n);
        const unsigned g = (ncell + 31) / 32;
        switch (scheme) {
        case AM_SCHEME_PBOX: octree_kernel<SCHEME_PBOX><<<g, 32, 0, s>>>(P); break;
        case AM_SCHEME_PBOX_AABB: octree_kernel<SCHEME_PBOX_AABB><<<g, 32, 0, s>>>(P); break;
        case AM_SCHEME_PICA: octree_kernel<SCHEME_PICA><<<g, 32, 0, s>>>(P); break;
        case AM_SCHEME_MICA: octree_kernel<SCHEME_MICA><<<g, 32, 0, s>>>(P); break;
        default: octree_kernel<SCHEME_AICA><<<g, 32, 0, s>>>(P); break;
        }
        if ((rc = kmark(ctx, s, AM_K_OCTREE))) return rc;
    }
    if (!dst_is_device)
        CK(cudaMemcpyAsync(am_out, gam, (size_t)ctx->MW * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    if ((rc = stream_end(ctx, s)) != AM_OK) return rc;
    if (stats) {
        unsigned long long h[4];
        CK(cudaMemcpyAsync(h, ctx->d_ostats, sizeof h, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        for (int k = 0; k < 4; ++k) stats[k] = (int64_t)h[k];
    } else if (!dst_is_device) {
        CK(cudaStreamSynchronize(s));
    }
    return AM_OK;
}

int am_unpack_cells(am_ctx* ctx, const uint32_t* words, uint8_t* cells, void* cuda_stream) {
    if (!ctx) return AM_EINVAL;
    if (!words || !cells) return fail(ctx, AM_EINVAL, "NULL buffer");
    DeviceGuard dg(ctx->device);
    const int nc = ctx->grid.m * ctx->grid.n;
    if (kchain(ctx, (cudaStream_t)cuda_stream)) return AM_ECUDA;
    unpack_cells_kernel<<<(nc + 255) / 256, 256, 0, (cudaStream_t)cuda_stream>>>(words, ctx->grid, cells);
    if (kmark(ctx, (cudaStream_t)cuda_stream, AM_K_LAYOUT)) return AM_ECUDA;
    CK(cudaGetLastError());
    return AM_OK;
}

int am_pack_cells(am_ctx* ctx, const uint8_t* cells, uint32_t* words, void* cuda_stream) {
    if (!ctx) return AM_EINVAL;
    if (!words || !cells) return fail(ctx, AM_EINVAL, "NULL buffer");
    DeviceGuard dg(ctx->device);
    if (kchain(ctx, (cudaStream_t)cuda_stream)) return AM_ECUDA;
    pack_cells_kernel<<<(ctx->MW + 255) / 256, 256, 0, (cudaStream_t)cuda_stream>>>(cells, ctx->grid, words);
    if (kmark(ctx, (cudaStream_t)cuda_stream, AM_K_LAYOUT)) return AM_ECUDA;
    CK(cudaGetLastError());
    return AM_OK;
}

int am_words_per_map(const am_ctx* ctx) { return ctx ? ctx->MW : -1; }

int64_t am_num_voxels(const am_ctx* ctx) { return ctx ? (int64_t)ctx->N : -1; }

const char* am_last_error(const am_ctx* ctx) {
    if (!ctx) return "NULL context";
    return ctx->err.empty() ? "no error" : ctx->err.c_str();
}

void am_destroy(am_ctx* ctx) {
    if (!ctx) return;
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(ctx->device);
    if (ctx->g_exec) cudaGraphExecDestroy(ctx->g_exec);
    if (ctx->cap_s) cudaStreamDestroy(ctx->cap_s);
    if (ctx->piv_ev) cudaEventDestroy(ctx->piv_ev);
    if (ctx->done_ev) cudaEventDestroy(ctx->done_ev);
    if (ctx->h_piv) cudaFreeHost(ctx->h_piv);
    for (int l = 0; l < kMaxLanes; ++l)
        if (ctx->lane_s[l]) cudaStreamDestroy(ctx->lane_s[l]);
    for (int l = 0; l <= kMaxLanes; ++l)
        if (ctx->lane_ev[l]) cudaEventDestroy(ctx->lane_ev[l]);
    cudaFree(ctx->d_vox);
    cudaFree(ctx->d_tab);
    cudaFree(ctx->d_am);
    cudaFree(ctx->d_ctr);
    cudaFree(ctx->d_queue);
    cudaFree(ctx->d_coarse);
    cudaFree(ctx->d_l1subs);
    cudaFree(ctx->d_live);
    cudaFree(ctx->d_live_full);
    cudaFree(ctx->d_recs);
    cudaFree(ctx->d_tasks);
    cudaFree(ctx->d_subs);
    cudaFree(ctx->d_supers);
    cudaFree(ctx->d_bricks);
    cudaFree(ctx->d_brick_list);
    cudaFree(ctx->d_texels);
    cudaFree(ctx->d_texels1);
    cudaFree(ctx->d_cmap);
    cudaFree(ctx->d_cmap_ones);
    cudaFree(ctx->d_prev);
    cudaFree(ctx->d_ts);
    cudaFree(ctx->d_piv);
    cudaFree(ctx->d_bctl);
    cudaFree(ctx->d_onode);
    cudaFree(ctx->d_olink);
    cudaFree(ctx->d_omemo);
    cudaFree(ctx->d_ostats);
    cudaFree(ctx->d_wit);
    cudaFree(ctx->d_hash);
    for (auto e : ctx->kev) cudaEventDestroy(e);
    for (auto e : ctx->ev_start) cudaEventDestroy(e);
    for (auto e : ctx->ev_stop) cudaEventDestroy(e);
    cudaGetLastError();
    if (prev >= 0) cudaSetDevice(prev);
    delete ctx;
}

}  // extern "C"
