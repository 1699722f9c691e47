// kernels.cuh -- shared device state and the non-streaming kernels of the AICA
// hot path on sm_100a: deferred band kernel, clear-direction map, all-pairs
// baseline kernel, upload helpers.  The voxel-streaming kernel is stream.cuh.
//
// Map of SURVEY.md 8(a) steps to code (kernel names as in am_kernel_name):
//   a1 voxel stream ........ batch.cuh bk_supers / bk_bricks / bk_voxels (kept 32-voxel
//                             sub-bricks, one warp each, coalesced LDG.128 with a
//                             streaming hint); stream.cuh filter_kernel reads every voxel
//                             (AM_OPT_BRICKS = 0)
//   a2 reach cull .......... stream.cuh fast_filter() / sphere_dropped(): D - r > rho_max
//   a3 cone axis ........... stream.cuh cone_of_voxel(): v, D, phi_v, gamma_v
//   a4 cone half-angles .... geometry.cuh tool_cones() / inner_cone()
//   a5 rasterise ........... stream.cuh raster_row(): per phi-row gamma intervals ->
//                             32-bit masks OR-ed into a per-CTA shared AM
//   a6 band resolution ..... band pairs pushed to a global queue; bk_band /
//                             band_exact_kernel run CHECKBOX only where the bit is still 0
//   a7 merge/flush/exit .... fused.cuh fused_flush(): one atomicOr per changed word;
//                             row-full bits skip full rows; a full map stops the later
//                             phases (early exit, am_stats.early_exit)
//   a8 output .............. bit-packed AM (layout in include/am.h)
//   a9 baseline ............ baseline_kernel: CHECKBOX for every (voxel, cell)
// The whole chain of one map runs as one cooperative launch (fused.cuh) or, for a
// batch of pivots, one launch per phase (batch.cuh).
#pragma once
#include <cstdint>

#include "geometry.cuh"

namespace am {

constexpr int kThreads = 256;
constexpr int kVPT = 4;                  // voxels per thread per tile (MLP for the HBM stream)
constexpr int kTile = kThreads * kVPT;   // voxels per tile

enum StatIdx {
    ST_STREAMED = 0, ST_CULLED, ST_SKIPPED, ST_LIVE, ST_ROWS, ST_BAND, ST_EXACT, ST_EXACT_HIT,
    ST_OVERFLOW, ST_EARLY, ST_PASSED, ST_ROWFULL, ST_COUNT
};

struct StreamParams {
    ToolDev tool;
    GridDev grid;
    float px, py, pz;
    const float4* __restrict__ vox;
    long long N;
    uint32_t* gam;                 // global AM, m * W words, zeroed before launch
    const float* __restrict__ tab; // cos phi[m], sin phi[m], cos gamma[n], sin gamma[n]
    unsigned long long* qcount;    // band queue fill counter (zeroed)
    unsigned long long* queue;     // band pairs: (voxel << 32) | cell
    long long qcap;
    unsigned long long* stats;     // ST_COUNT counters (zeroed)
    unsigned long long* early;     // the map's early-exit flag (main stats[ST_EARLY]): set once the map
                                   // is full; every later phase of that map then returns at once (a7)
    int refresh_tiles;
    // band-queue voxel references: bit 31 of the queued index selects vox_coarse
    const float4* __restrict__ vox_main;
    const float4* __restrict__ vox_coarse;
    unsigned int vtag;             // OR-ed into queued indices by this launch
    unsigned int vbase;            // index of vox[0] within its array
    // clear-direction map: per texel (cos, sin) of the angle from
    // its centre to the nearest cell still clear, rounded down; the texel centres of that map
    const float4* __restrict__ cmap;
    const float4* __restrict__ cmap_tex;
    int cmapT;                     // texels per cube-face side
    float cull_dist;               // rho_max, grown by the fp32 guard (reach cull)
    unsigned int* live_count;      // live voxels found by the filter (zeroed; may exceed live_cap)
    unsigned int* live_idx;        // their indices into vox, the first live_cap of them
    unsigned int live_cap;         // capacity of live_idx; a live voxel past it is rasterised inline (exact)
    int may_cull;                  // some voxel may lie beyond the tool's reach (per pivot)
    // cone records and (voxel, row) tasks between cone_kernel and row_kernel
    struct ConeRec* recs;
    unsigned long long* tasks;     // (record << 16) | row offset
    unsigned int* rec_count;       // zeroed per launch pair
    unsigned long long* task_count;
    unsigned int rec_cap;
    unsigned long long task_cap;
    // bricks of kThreads consecutive voxels of vox: bounding spheres (x, y, z, r)
    const float4* __restrict__ bricks;
    unsigned int nbricks;
    unsigned int* brick_list;      // bricks kept by brick_test_kernel (capacity nbricks)
    unsigned int* brick_count;     // zeroed per map
    int band_vdepth;               // band pairs: virtual sub-cube levels before CHECKBOX (§4.3)
    // AM reuse between neighbouring pivots (AM_OPT_REUSE; 8(f) NEXT 2): per cell of this
    // map, the id of a voxel whose inner cone set it (nullptr: off; ids: bit 31 = coarse array).  The
    // slot's next map rasterises the inner cones of these witnesses -- at its own pivot, so exactly --
    // with level 0
    unsigned int* wit;
    // sub-bricks of 32 consecutive voxels (one warp of a brick): bounding spheres;
    // nullptr = not tested
    const float4* __restrict__ subs;
    // super-bricks of 8 bricks (batched path): bounding spheres (nullptr = not tested),
    // kept super-bricks of this map and their count (zeroed per map)
    const float4* __restrict__ supers;
    unsigned int* super_list;
    unsigned int* super_count;
};

// Cube-map texel of direction v (any length): face = dominant axis and sign,
// (u, w) = the other two components over the dominant one.  The host computes
// each texel's centre and an angular radius that bounds every direction this
// exact function maps into the texel.
__device__ __forceinline__ int cube_texel(float vx, float vy, float vz, int T) {
    const float ax = fabsf(vx), ay = fabsf(vy), az = fabsf(vz);
    const bool xm = ax >= fmaxf(ay, az);
    const bool ym = !xm && ay >= az;
    const float a = fmaxf(ax, fmaxf(ay, az));
    const float u = xm ? vy : vx;
    const float w = (xm || ym) ? vz : vy;
    const int face = xm ? (vx < 0.f) : (ym ? 2 + (vy < 0.f) : 4 + (vz < 0.f));
    const float hs = 0.5f * (float)T;
    const float s = hs * __frcp_rn(a);
    const int iu = min(T - 1, max(0, __float2int_rz(fmaf(u, s, hs))));
    const int iw = min(T - 1, max(0, __float2int_rz(fmaf(w, s, hs))));
    return (face * T + iw) * T + iu;
}

__device__ __forceinline__ uint32_t ld_cg(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

__device__ __forceinline__ uint32_t ld_vol_shared(const uint32_t* p) {
    return *reinterpret_cast<const volatile uint32_t*>(p);
}

__device__ __forceinline__ uint32_t row_word_mask(int w, int n) {
    const int rem = n - (w << 5);
    return rem >= 32 ? 0xffffffffu : ((1u << rem) - 1u);
}

// Exact test of one (voxel, cell) pair with directions from the global tables.
__device__ __forceinline__ bool exact_pair(const StreamParams& p, float4 q, int cell) {
    const int i = cell / p.grid.n, j = cell - i * p.grid.n;
    const float* t = p.tab;
    const float cph = __ldg(t + i), sph = __ldg(t + p.grid.m + i);
    const float cg = __ldg(t + 2 * p.grid.m + j), sg = __ldg(t + 2 * p.grid.m + p.grid.n + j);
    if (p.band_vdepth > 0) {  // PAPER.md §4.3: virtual children by CHECKICA first
        unsigned int nb = 0, ni = 0;
        return leaf_expand(q.x - p.px, q.y - p.py, q.z - p.pz, q.w, sph * cg, sph * sg, cph, p.band_vdepth, p.tool,
                           nb, ni);
    }
    return exact_hit(q.x - p.px, q.y - p.py, q.z - p.pz, q.w, sph * cg, sph * sg, cph, p.tool);
}

// Cold-path counters of one CTA, kept in shared memory (32-bit; flushed to the
// 64-bit global stats when the CTA retires) so they cost no registers.
struct Counters {
    unsigned int* c;  // [CT_LIVE, CT_ROWS, CT_BAND, CT_OVERFLOW]
};
enum { CT_LIVE = 0, CT_ROWS, CT_BAND, CT_OVERFLOW, CT_ROWFULL, CT_COUNT };

// Are all rows i0..i1 full (bit set in sRowFull)?
__device__ __forceinline__ bool rows_all_full(const uint32_t* sRowFull, int i0, int i1) {
    for (int w = i0 >> 5; w <= (i1 >> 5); ++w) {
        uint32_t need = 0xffffffffu;
        if (w == (i0 >> 5)) need &= 0xffffffffu << (i0 & 31);
        if (w == (i1 >> 5)) need &= 0xffffffffu >> (31 - (i1 & 31));
        if ((ld_vol_shared(sRowFull + w) & need) != need) return false;
    }
    return true;
}

__device__ void fill_all(const StreamParams& p, uint32_t* sAM) {
    const int W = p.grid.W;
    for (int i = 0; i < p.grid.m; ++i)
        for (int w = 0; w < W; ++w) atomicOr(sAM + i * W + w, row_word_mask(w, p.grid.n));
}

__device__ __forceinline__ void push_band(const StreamParams& p, uint32_t* sAM, unsigned int vidx,
                                          float4 q, int cell, uint32_t* wp, uint32_t bit,
                                          Counters& cnt) {
    if (cnt.c) atomicAdd(cnt.c + CT_BAND, 1u);
    const unsigned long long slot = atomicAdd(p.qcount, 1ULL);
    if ((long long)slot < p.qcap) {
        p.queue[slot] = ((unsigned long long)vidx << 32) | (unsigned int)cell;
    } else {
        // queue full: resolve inline (rare; keeps the result exact)
        if (cnt.c) atomicAdd(cnt.c + CT_OVERFLOW, 1u);
        if (exact_pair(p, q, cell)) atomicOr(wp, bit);
    }
}

// (the voxel-streaming kernel lives in stream.cuh)

// Clear-direction map: for every cube-map texel t with centre c_t
// and angular radius r_t, U_t >= cos(max(0, angle(c_t, nearest clear cell) - r_t)),
// so any direction mapped to t is at least acos(U_t) away from every cell that
// is still clear in `gam`; U_t = -2 when no cell is clear.  The map stores
// V_t = U_t |U_t| (monotone in U; lets the filter compare squared cosines).
// Cells only ever get blocked, so a map built from a partial AM stays valid
// for the final one.
//
//
// Texels are processed in 4 x 4 blocks ("coarse texels", one warp each): the
// warp first finds the coarse centre's nearest clear angle theta_C over every
// clear direction, then only directions within theta_C + 2 rho of the coarse
// centre (rho = the block's angular radius) can be nearest to any of its 16
// texels (triangle inequality), and only those are tried per texel.  With few
// clear cells (the common case once the coarse levels are in: ~100 of 4096 at
// C3), more than fit in shared memory, or T not a multiple of 4, every texel
// tries every clear direction (in chunks), 4 texels per thread.

constexpr int kMapDirs = 2048;  // clear directions staged in shared memory per chunk

__device__ __forceinline__ float dot3(float4 a, float4 b) { return fmaf(a.x, b.x, fmaf(a.y, b.y, a.z * b.z)); }

// V_t from the best cosine of texel (c, r): the nearest-cell angle rounded
// down and the bound rounded up (fp32 guards).
__device__ __forceinline__ float4 clear_map_value(float best, float r) {
    // (cos theta, sin theta, U_t |U_t|, 0): theta = the texel centre's nearest-clear angle, cos
    // rounded up (theta down); U_t = cos(max(0, theta - r)) bounds every direction of the texel
    // (r = its radius), evaluated as b cos r + sin theta sin r without acos/cos (the fast sin/cos
    // and square-root errors, < 1e-6, are inside the guard).  No clear cell: (-2, 0, -4, 0).
    if (best < -1.5f) return make_float4(-2.f, 0.f, -4.f, 0.f);
    const float b = fminf(best + 2e-6f, 1.f);
    const float st = sqrtf(fmaxf((1.f - b) * (1.f + b), 0.f));
    const float cr = __cosf(r), sr = __sinf(r);
    const float u = (b >= cr) ? 1.f : fminf(fmaf(b, cr, st * sr) + 4e-6f, 1.f);
    return make_float4(b, st, u * fabsf(u), 0.f);
}

// Compact the directions of the clear cells of words [w0, w1) of sAM into
// sDirs (at most kMapDirs: the caller sizes the range); count in *sN.
__device__ void compact_clear_dirs(const uint32_t* sAM, const GridDev& g, const float* __restrict__ tab, int w0,
                                   int w1, float4* sDirs, int* sN) {
    __syncthreads();
    if (threadIdx.x == 0) *sN = 0;
    __syncthreads();
    for (int w = w0 + threadIdx.x; w < w1; w += blockDim.x) {
        const int i = w / g.W, wj = w - i * g.W;
        uint32_t clear = ~sAM[w] & row_word_mask(wj, g.n);
        if (!clear) continue;
        int pos = atomicAdd(sN, __popc(clear));
        const float cph = __ldg(tab + i), sph = __ldg(tab + g.m + i);
        while (clear) {
            const int j = (wj << 5) + __ffs(clear) - 1;
            clear &= clear - 1u;
            sDirs[pos++] = make_float4(sph * __ldg(tab + 2 * g.m + j), sph * __ldg(tab + 2 * g.m + g.n + j), cph, 0.f);
        }
    }
    __syncthreads();
}

// Row-ordered nearest-clear search (the clear map's large-count path).  For a
// direction c = (sin phi_c cos g_c, sin phi_c sin g_c, cos phi_c) and a cell of
// row i, cos angle = cos phi_i cos phi_c + sin phi_i sin phi_c cos(g_j - g_c):
// both sines are >= 0 (phi in (0, pi)), so within a row the best cell is the
// clear cell nearest to g_c in circular gamma -- the first clear cell at or
// after g_c or the last one before it -- and no cell of row i can beat
// ub_i = cos(phi_i - phi_c).  Rows are visited from phi_c outward (ub
// decreasing in each direction, larger ub first) and the search stops once both
// directions' ub fall below the best cosine found.  Result: the maximum of
// c . d over the clear cells, as the all-pairs loop computes it, up to fp32
// rounding of the same dot products (absorbed by clear_map_value's guards).
// clr: per-row clear masks (W words per row, padding bits 0); rows: one bit per
// row with a clear cell.
__device__ __forceinline__ int next_row_at_or_after(const uint32_t* rows, int i, int m) {
    if (i >= m) return m;
    int w = i >> 5;
    uint32_t x = rows[w] & (0xffffffffu << (i & 31));
    const int RW = (m + 31) >> 5;
    while (!x) {
        if (++w >= RW) return m;
        x = rows[w];
    }
    return (w << 5) + __ffs(x) - 1;
}

__device__ __forceinline__ int prev_row_at_or_before(const uint32_t* rows, int i) {
    if (i < 0) return -1;
    int w = i >> 5;
    uint32_t x = rows[w] & (0xffffffffu >> (31 - (i & 31)));
    while (!x) {
        if (--w < 0) return -1;
        x = rows[w];
    }
    return (w << 5) + 31 - __clz(x);
}

__device__ __forceinline__ float row_best_cos(float4 c, const uint32_t* clr, int i, int j0, const GridDev& g,
                                              const float* __restrict__ tab) {
    const int W = g.W, n = g.n;
    const uint32_t* row = clr + i * W;
    // first clear cell at or after j0 (circular; the row has one)
    int w = j0 >> 5;
    uint32_t x = row[w] & (0xffffffffu << (j0 & 31));
    while (!x) {
        w = (w + 1 == W) ? 0 : w + 1;
        x = row[w];
    }
    const int jr = (w << 5) + __ffs(x) - 1;
    // last clear cell at or before j0 - 1 (circular)
    const int jl0 = j0 == 0 ? n - 1 : j0 - 1;
    w = jl0 >> 5;
    x = row[w] & (0xffffffffu >> (31 - (jl0 & 31)));
    while (!x) {
        w = (w == 0) ? W - 1 : w - 1;
        x = row[w];
    }
    const int jl = (w << 5) + 31 - __clz(x);
    const float cph = __ldg(tab + i), sph = __ldg(tab + g.m + i);
    const float* cg = tab + 2 * g.m;
    const float* sg = cg + n;
    const float br = fmaf(cph, c.z, sph * fmaf(c.x, __ldg(cg + jr), c.y * __ldg(sg + jr)));
    const float bl = fmaf(cph, c.z, sph * fmaf(c.x, __ldg(cg + jl), c.y * __ldg(sg + jl)));
    return fmaxf(br, bl);
}

__device__ float nearest_clear_rows(float4 c, const uint32_t* clr, const uint32_t* rows, const GridDev& g,
                                    const float* __restrict__ tab) {
    const int m = g.m, n = g.n;
    const float cz = fminf(fmaxf(c.z, -1.f), 1.f);
    const float sc = sqrtf(fmaf(c.x, c.x, c.y * c.y));
    const float phic = acosf(cz);
    float gc = atan2f(c.y, c.x);
    if (gc < 0.f) gc += 6.2831853071795865f;
    int j0 = (int)ceilf(fmaf(gc, g.inv_dgam, -0.5f));
    j0 = j0 < 0 ? 0 : (j0 >= n ? 0 : j0);
    // row ic: phi_ic <= phi_c < phi_ic+1 (up to rounding: ub is then non-monotone only at rounding level)
    const int ic = min(m - 1, max(-1, (int)floorf(fmaf(phic, g.inv_dphi, -0.5f))));
    int id = prev_row_at_or_before(rows, ic);
    int iu = next_row_at_or_after(rows, ic + 1, m);
    float best = -2.f;
    for (;;) {
        const float ud = id >= 0 ? fmaf(__ldg(tab + id), cz, __ldg(tab + m + id) * sc) : -3.f;
        const float uu = iu < m ? fmaf(__ldg(tab + iu), cz, __ldg(tab + m + iu) * sc) : -3.f;
        const bool down = ud >= uu;
        const float ub = down ? ud : uu;
        if (ub < best - 1e-6f || ub < -2.5f) break;
        const int i = down ? id : iu;
        best = fmaxf(best, row_best_cos(c, clr, i, j0, g, tab));
        if (down)
            id = prev_row_at_or_before(rows, id - 1);
        else
            iu = next_row_at_or_after(rows, iu + 1, m);
    }
    return best;
}

// The cells still clear in sAM as directions in sDirs, by the whole CTA; returns
// their count, or -1 (and no list) when there are more than kMapDirs.
__device__ int clear_list_cta(const uint32_t* sAM, const GridDev& g, const float* __restrict__ tab, float4* sDirs,
                              int* sN) {
    const int MW = g.m * g.W;
    __syncthreads();
    if (threadIdx.x == 0) *sN = 0;
    __syncthreads();
    int cnt = 0;
    for (int w = threadIdx.x; w < MW; w += blockDim.x) cnt += __popc(~sAM[w] & row_word_mask(w % g.W, g.n));
    if (cnt) atomicAdd(sN, cnt);
    __syncthreads();
    const int total = *sN;
    if (total > kMapDirs) return -1;
    compact_clear_dirs(sAM, g, tab, 0, MW, sDirs, sN);
    return total;
}

// The cells still clear in sAM as directions in sDirs in row-major order, with
// sRowStart[i] = index of row i's first (sRowStart[m] = the count), by the
// whole CTA; returns the count, or -1 (no list) when there are more than
// kMapDirs.  A cone that spans rows a0..a1 only needs [sRowStart[a0], sRowStart[a1 + 1]).
__device__ int clear_list_rows_cta(const uint32_t* sAM, const GridDev& g, const float* __restrict__ tab,
                                   float4* sDirs, int* sRowStart) {
    const int m = g.m, W = g.W;
    __syncthreads();
    for (int i = threadIdx.x; i < m; i += blockDim.x) {
        int c = 0;
        for (int w = 0; w < W; ++w) c += __popc(~sAM[i * W + w] & row_word_mask(w, g.n));
        sRowStart[i + 1] = c;
    }
    if (threadIdx.x == 0) sRowStart[0] = 0;
    __syncthreads();
    if (threadIdx.x < 32) {  // prefix sums: each lane a chunk of rows, then a warp scan of the chunk sums
        const int lane = threadIdx.x, per = (m + 31) >> 5;
        const int b = 1 + lane * per, e = min(m + 1, b + per);
        int sum = 0;
        for (int k = b; k < e; ++k) sum += sRowStart[k];
        int incl = sum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int t = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += t;
        }
        int run = incl - sum;
        for (int k = b; k < e; ++k) {
            run += sRowStart[k];
            sRowStart[k] = run;
        }
    }
    __syncthreads();
    const int total = sRowStart[m];
    if (total > kMapDirs) return -1;
    for (int i = threadIdx.x; i < m; i += blockDim.x) {
        int pos = sRowStart[i];
        const float cph = __ldg(tab + i), sph = __ldg(tab + m + i);
        for (int w = 0; w < W; ++w) {
            uint32_t clear = ~sAM[i * W + w] & row_word_mask(w, g.n);
            while (clear) {
                const int j = (w << 5) + __ffs(clear) - 1;
                clear &= clear - 1u;
                sDirs[pos++] = make_float4(sph * __ldg(tab + 2 * m + j), sph * __ldg(tab + 2 * m + g.n + j), cph, 0.f);
            }
        }
    }
    __syncthreads();
    return total;
}

// Coarse-block path for B x B texel blocks (B = 8), one warp per block:
// lane l holds the texels (l % B, l / B + k 32/B), k < B^2/32.  The block centre
// c (normalised sum of its texel centres) and radius rho (max angle from c to
// a texel centre, rounded up) bound the search: with theta_C = the angle from
// c to its nearest clear direction, every texel's nearest clear direction lies
// within theta_C + 2 rho of c (triangle inequality), so only those candidates
// (found by one ballot pass over the list) are tried per texel.  c and
// cos / sin(2 rho + slack) come from the host-made block table after the texels.
__device__ void clear_map_blocks(const float4* __restrict__ texels, int T, float4* __restrict__ V,
                                 const float4* sDirs, int total, int w0, int wstride, float far_cos = -2.f) {
    constexpr int B = 8, TPL = B * B / 32, ROWS = 32 / B;
    const int lane = threadIdx.x & 31;
    const int Tc = T / B, nct = 6 * Tc * Tc;
    const float inv1 = 1.f / (float)(Tc * Tc), inv2 = 1.f / (float)Tc;
    const float4* __restrict__ blocks = texels + 6 * T * T;  // host-made block table (am.cu make_texels)
    for (int ct = w0; ct < nct; ct += wstride) {
        // (ct < 2^22: the float quotients floor exactly)
        const int face = (int)(((float)ct + 0.5f) * inv1), rem = ct - face * Tc * Tc;
        const int cw = (int)(((float)rem + 0.5f) * inv2), cu = rem - cw * Tc;
        const int t0 = (face * T + B * cw + lane / B) * T + B * cu + lane % B;
        float4 f[TPL];
#pragma unroll
        for (int k = 0; k < TPL; ++k) f[k] = texels[t0 + k * ROWS * T];
        const float4 A = blocks[2 * ct];   // block centre c, cos(2 rho')
        const float sR = blocks[2 * ct + 1].x;  // sin(2 rho')
        const float4 c = make_float4(A.x, A.y, A.z, 0.f);
        float bc = -2.f;
        for (int e = lane; e < total; e += 32) bc = fmaxf(bc, dot3(c, sDirs[e]));
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) bc = fmaxf(bc, __shfl_xor_sync(0xffffffffu, bc, o));
        if (bc < far_cos) {  // (warp-uniform) a far block: no per-texel search
            // every clear cell is at least theta_C from c, so at least theta_C - a_t from texel centre t
            // (a_t = angle(t, c) <= rho < theta_C; triangle inequality): store that lower bound,
            // cos(theta_C - a_t) = cos theta_C cos a_t + sin theta_C sin a_t, with theta_C and a_t rounded
            // down / up by 1e-6 in the cosine and the result rounded up
            const float bg = fminf(bc + 1e-6f, 1.f);
            const float sb = sqrtf(fmaxf((1.f - bg) * (1.f + bg), 0.f));
#pragma unroll
            for (int k = 0; k < TPL; ++k) {
                const float ca = fmaxf(dot3(f[k], c) - 1e-6f, -1.f);
                const float sa = sqrtf(fmaxf((1.f - ca) * (1.f + ca), 0.f));
                V[t0 + k * ROWS * T] = clear_map_value(fminf(fmaf(bg, ca, sb * sa) + 1e-6f, 1.f), f[k].w);
            }
            continue;
        }
        // thr = cos(theta_C' + 2 rho') - 1e-6 with cos theta_C' = b (rounded down): the sum
        // formula, sin theta_C' = sqrt((1 - b)(1 + b)); -2 (every candidate) past pi
        const float b = fmaxf(bc - 1e-6f, -1.f);
        const float thr = (b <= -A.w) ? -2.f
                                      : fmaf(b, A.w, -sqrtf(fmaxf((1.f - b) * (1.f + b), 0.f)) * sR) - 1e-6f;
        float bf[TPL];
#pragma unroll
        for (int k = 0; k < TPL; ++k) bf[k] = -2.f;
        for (int base = 0; base < total; base += 32) {
            const int e = base + lane;
            unsigned int mask = __ballot_sync(0xffffffffu, e < total && dot3(c, sDirs[e]) >= thr);
            while (mask) {  // two candidates per pass (the second repeats the first when alone)
                const int k1 = __ffs(mask) - 1;
                mask &= mask - 1u;
                const int k2 = mask ? __ffs(mask) - 1 : k1;
                mask &= mask - 1u;
                const float4 d1 = sDirs[base + k1], d2 = sDirs[base + k2];
#pragma unroll
                for (int k = 0; k < TPL; ++k) bf[k] = fmaxf(bf[k], fmaxf(dot3(f[k], d1), dot3(f[k], d2)));
            }
        }
#pragma unroll
        for (int k = 0; k < TPL; ++k) V[t0 + k * ROWS * T] = clear_map_value(bf[k], f[k].w);
    }
}

// The clear-direction map of `gam` into V (6 T^2 texels), computed by the CTAs
// gb = 0..gn-1 of a group.  Shared memory: sAM (m * W words), sDirs
// (kMapDirs), sN.
__device__ int clear_map_cta(const uint32_t* gam, const GridDev& g, const float* __restrict__ tab,
                              const float4* __restrict__ texels, int T, float4* __restrict__ V, uint32_t* sAM,
                              float4* sDirs, int* sN, unsigned int gb, unsigned int gn, bool warp_texel = false,
                              bool final_map = false) {
    const int MW = g.m * g.W;
    const int ntex = 6 * T * T;
    __syncthreads();
    if (threadIdx.x == 0) *sN = 0;
    __syncthreads();
    int cnt = 0;
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        const uint32_t a = ld_cg(gam + w);
        sAM[w] = a;
        cnt += __popc(~a & row_word_mask(w % g.W, g.n));
    }
    if (cnt) atomicAdd(sN, cnt);
    __syncthreads();
    const int total = *sN;
    if (total == 0) return 0;  // the map is full (early exit): no clear cell to find
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    // few texels for the grid's warps (the map after level 0 of ONE pivot): one WARP per texel, the
    // lanes share the clear directions (the same maximum as every other path)
    if (warp_texel && total <= kMapDirs && ntex <= 4 * (int)(gn * nwarps)) {
        compact_clear_dirs(sAM, g, tab, 0, MW, sDirs, sN);
        for (int t = gb * nwarps + warp; t < ntex; t += gn * nwarps) {
            const float4 c = texels[t];
            float best = -2.f;
            for (int e = lane; e < total; e += 32) best = fmaxf(best, dot3(c, sDirs[e]));
            best = fmaxf(best, __shfl_xor_sync(0xffffffffu, best, 16));
            best = fmaxf(best, __shfl_xor_sync(0xffffffffu, best, 8));
            best = fmaxf(best, __shfl_xor_sync(0xffffffffu, best, 4));
            best = fmaxf(best, __shfl_xor_sync(0xffffffffu, best, 2));
            best = fmaxf(best, __shfl_xor_sync(0xffffffffu, best, 1));
            if (lane == 0) V[t] = clear_map_value(best, c.w);
        }
        return total;
    }
#ifndef AM_ROWSCAN_OVER_DIRS
#define AM_ROWSCAN_OVER_DIRS 1
#endif
    // (more clear cells than fit in shared memory: clear cells are dense, so the
    // row-ordered nearest-clear search stops after a few rows)
    if (total > g.rowscan || (AM_ROWSCAN_OVER_DIRS && total > kMapDirs)) {
        // clear masks in place (sAM is re-seeded by every caller before reuse),
        // one bit per row with a clear cell in the sDirs space
        uint32_t* sRows = reinterpret_cast<uint32_t*>(sDirs);
        for (int w = threadIdx.x; w < ((g.m + 31) >> 5); w += blockDim.x) sRows[w] = 0u;
        __syncthreads();
        for (int w = threadIdx.x; w < MW; w += blockDim.x) {
            const int i = w / g.W;
            const uint32_t cl = ~sAM[w] & row_word_mask(w - i * g.W, g.n);
            sAM[w] = cl;
            if (cl) atomicOr(sRows + (i >> 5), 1u << (i & 31));
        }
        __syncthreads();
        for (int t = gb * blockDim.x + threadIdx.x; t < ntex; t += gn * blockDim.x) {
            const float4 c = texels[t];
            V[t] = clear_map_value(nearest_clear_rows(c, sAM, sRows, g, tab), c.w);
        }
        return total;
    }
#ifndef AM_MAP1_BLOCK4
#define AM_MAP1_BLOCK4 1  // the map after level 0 (not final_map) by 4x4 texel blocks (r5_sweeps.txt)
#endif
    if (total > g.brute && total <= kMapDirs && g.cblock == 8 && (T & 7) == 0 && !(AM_MAP1_BLOCK4 && !final_map)) {
        compact_clear_dirs(sAM, g, tab, 0, MW, sDirs, sN);
        // (the far-block bound only for the final map: its blocks are small, rho ~ 4 deg at T = 96, where
        //  the map after level 0, T1 = 16, would give up to 2 rho ~ 60 deg per texel)
        clear_map_blocks(texels, T, V, sDirs, total, gb * nwarps + warp, gn * nwarps, final_map ? g.far_cos : -2.f);
        return total;
    }
    if (total > g.brute && total <= kMapDirs && (T & 3) == 0) {
        compact_clear_dirs(sAM, g, tab, 0, MW, sDirs, sN);
        const int Tc = T >> 2, nct = 6 * Tc * Tc;
        const int half = lane >> 4, sub = lane & 15;
        for (int ct = gb * nwarps + warp; ct < nct; ct += gn * nwarps) {
            const int face = ct / (Tc * Tc), rem = ct - face * Tc * Tc, cw = rem / Tc, cu = rem - cw * Tc;
            const int t = (face * T + 4 * cw + (sub >> 2)) * T + 4 * cu + (sub & 3);
            const float4 cf = texels[t];
            // coarse centre: the normalised sum of the 16 texel centres (each half-warp)
            float sx = cf.x, sy = cf.y, sz = cf.z;
#pragma unroll
            for (int o = 1; o < 16; o <<= 1) {
                sx += __shfl_xor_sync(0xffffffffu, sx, o);
                sy += __shfl_xor_sync(0xffffffffu, sy, o);
                sz += __shfl_xor_sync(0xffffffffu, sz, o);
            }
            const float inv = rsqrtf(fmaf(sx, sx, fmaf(sy, sy, sz * sz)));
            const float4 c = make_float4(sx * inv, sy * inv, sz * inv, 0.f);
            // rho: block radius (angles rounded up)
            float rho = acosf(fmaxf(dot3(cf, c) - 1e-6f, -1.f));
#pragma unroll
            for (int o = 1; o < 16; o <<= 1) rho = fmaxf(rho, __shfl_xor_sync(0xffffffffu, rho, o));
            // theta_C over every clear direction
            float bc = -2.f;
            for (int e = lane; e < total; e += 32) bc = fmaxf(bc, dot3(c, sDirs[e]));
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) bc = fmaxf(bc, __shfl_xor_sync(0xffffffffu, bc, o));
            // candidates: angle(c, d) <= theta_C + 2 rho (rounded up, + slack)
            const float th = acosf(fmaxf(bc - 1e-6f, -1.f)) + 2.f * rho + 1e-4f;
            const float thr = th >= 3.14159f ? -2.f : cosf(th) - 1e-6f;
            float bf = -2.f;
            for (int base = 0; base < total; base += 32) {
                const int e = base + lane;
                unsigned int mask = __ballot_sync(0xffffffffu, e < total && dot3(c, sDirs[e]) >= thr);
                while (mask) {  // half-warps take alternate candidates
                    const int k0 = __ffs(mask) - 1;
                    mask &= mask - 1u;
                    int k = half ? -1 : k0;
                    if (mask) {
                        if (half) k = __ffs(mask) - 1;
                        mask &= mask - 1u;
                    }
                    if (k >= 0) bf = fmaxf(bf, dot3(cf, sDirs[base + k]));
                }
            }
            bf = fmaxf(bf, __shfl_xor_sync(0xffffffffu, bf, 16));
            if (!half) V[t] = clear_map_value(bf, cf.w);
        }
        return total;
    }
    // every texel against every clear direction, kMaxT texels per thread per
    // pass, the directions in chunks of whole words
    constexpr int kMaxT = 4;
    const int per_pass = kMaxT * gn * blockDim.x;
    for (int t0 = 0; t0 < ntex; t0 += per_pass) {
        float best[kMaxT];
        float4 c[kMaxT];
#pragma unroll
        for (int j = 0; j < kMaxT; ++j) {
            best[j] = -2.f;
            const int t = t0 + (j * gn + gb) * blockDim.x + threadIdx.x;
            c[j] = t < ntex ? texels[t] : make_float4(0.f, 0.f, 1.f, 0.f);
        }
        for (int w0 = 0; w0 < MW; w0 += kMapDirs / 32) {
            compact_clear_dirs(sAM, g, tab, w0, min(MW, w0 + kMapDirs / 32), sDirs, sN);
            const int k = *sN;
            for (int e = 0; e < k; ++e) {
                const float4 d = sDirs[e];
#pragma unroll
                for (int j = 0; j < kMaxT; ++j) best[j] = fmaxf(best[j], dot3(c[j], d));
            }
        }
#pragma unroll
        for (int j = 0; j < kMaxT; ++j) {
            const int t = t0 + (j * gn + gb) * blockDim.x + threadIdx.x;
            if (t < ntex) V[t] = clear_map_value(best[j], c[j].w);
        }
    }
    return total;
}

// Stand-alone launch of clear_map_cta (multi-kernel path); dynamic shared
// memory: m * W words, then kMapDirs float4 (16-byte aligned).
__host__ __device__ inline size_t clear_map_smem_bytes(int MW) {
    return (((size_t)MW * sizeof(uint32_t) + 15) & ~(size_t)15) + (size_t)kMapDirs * sizeof(float4);
}

__global__ void __launch_bounds__(256) clear_map_kernel(const uint32_t* __restrict__ gam, GridDev g,
                                                        const float* __restrict__ tab,
                                                        const float4* __restrict__ texels, int T,
                                                        float4* __restrict__ V, unsigned long long* early) {
    extern __shared__ __align__(16) unsigned char smem_cm[];
    __shared__ int sN;
    uint32_t* sAM = reinterpret_cast<uint32_t*>(smem_cm);
    float4* sDirs = reinterpret_cast<float4*>(smem_cm + (((size_t)g.m * g.W * sizeof(uint32_t) + 15) & ~(size_t)15));
    const int total = clear_map_cta(gam, g, tab, texels, T, V, sAM, sDirs, &sN, blockIdx.x, gridDim.x);
    if (total == 0 && early && blockIdx.x == 0 && threadIdx.x == 0) *early = 1ull;
}

// Early exit (a7, SURVEY 8(a) "stop when popcount(AM) = m n"): has a clear-map phase of this
// map found it full?  One read per CTA, broadcast through shared memory, so every thread of the
// CTA takes the same branch even while another CTA of the same launch is setting the flag (the
// map launch sets it while its own CTAs may still be starting).  Every thread must call it.
__device__ __forceinline__ bool map_full(const unsigned long long* early) {
    __shared__ int s_full;
    __syncthreads();  // (a previous call's readers are done with s_full)
    if (threadIdx.x == 0) s_full = early && *reinterpret_cast<const volatile unsigned long long*>(early) != 0ull;
    __syncthreads();
    return s_full != 0;
}

// a6: exact test for queued band pairs whose AM bit is still clear.
__global__ void __launch_bounds__(kThreads) band_exact_kernel(const StreamParams p) {
    if (map_full(p.early)) return;
    const unsigned long long cnt = *p.qcount;
    const long long n = (long long)(cnt < (unsigned long long)p.qcap ? cnt : (unsigned long long)p.qcap);
    if ((long long)blockIdx.x * blockDim.x >= n) return;  // (whole CTA: nothing queued for it)
    unsigned long long tests = 0, hits = 0;
    for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < n;
         k += (long long)gridDim.x * blockDim.x) {
        const unsigned long long e = p.queue[k];
        const unsigned int vidx = (unsigned int)(e >> 32);
        const int cell = (int)(e & 0xffffffffu);
        const int i = cell / p.grid.n, j = cell - i * p.grid.n;
        uint32_t* wp = p.gam + i * p.grid.W + (j >> 5);
        const uint32_t bit = 1u << (j & 31);
        if (ld_cg(wp) & bit) continue;
        ++tests;
        const float4 q = (vidx & 0x80000000u) ? p.vox_coarse[vidx & 0x7fffffffu] : p.vox_main[vidx];
        if (exact_pair(p, q, cell)) {
            ++hits;
            atomicOr(wp, bit);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        tests += __shfl_xor_sync(0xffffffffu, tests, o);
        hits += __shfl_xor_sync(0xffffffffu, hits, o);
    }
    if ((threadIdx.x & 31) == 0) {
        if (tests) atomicAdd(p.stats + ST_EXACT, tests);
        if (hits) atomicAdd(p.stats + ST_EXACT_HIT, hits);
    }
}

// a9: baseline -- CHECKBOX for every (voxel, cell) pair, one CTA per cell,
// stopping at the first collision (Alg. 2).  `reject` enables an
// exact-safe bounding-sphere reject (circumscribed ball vs each cylinder).
__global__ void __launch_bounds__(kThreads) baseline_kernel(const StreamParams p, int reject) {
    const int ncell = p.grid.m * p.grid.n;
    for (int cell = blockIdx.x; cell < ncell; cell += gridDim.x) {
        const int i = cell / p.grid.n, j = cell - i * p.grid.n;
        const float cph = __ldg(p.tab + i), sph = __ldg(p.tab + p.grid.m + i);
        const float cg = __ldg(p.tab + 2 * p.grid.m + j), sg = __ldg(p.tab + 2 * p.grid.m + p.grid.n + j);
        const float dx = sph * cg, dy = sph * sg, dz = cph;
        int found = 0;
        for (long long b = 0; b < p.N; b += blockDim.x) {
            const long long idx = b + threadIdx.x;
            int hit = 0;
            if (idx < p.N) {
                const float4 q = __ldg(p.vox + idx);
                const float vx = q.x - p.px, vy = q.y - p.py, vz = q.z - p.pz;
                bool cand = true;
                if (reject) {
                    // circumscribed ball (grown) vs each cylinder, 2-D meridian distance
                    const float a = vx * dx + vy * dy + vz * dz;
                    const float ex = vx - a * dx, ey = vy - a * dy, ez = vz - a * dz;
                    const float rho = sqrtf(ex * ex + ey * ey + ez * ez);
                    const float r2 = kSqrt3 * q.w * (1.f + 1e-5f) + 1e-5f * (fabsf(a) + rho);
                    cand = false;
                    for (int k = 0; k < p.tool.ncyl; ++k) {
                        const float da = a < p.tool.z0[k] ? p.tool.z0[k] - a
                                                          : (a > p.tool.z1[k] ? a - p.tool.z1[k] : 0.f);
                        const float dr = fmaxf(rho - p.tool.R[k], 0.f);
                        if (da * da + dr * dr <= r2 * r2) cand = true;
                    }
                }
                hit = cand && exact_hit(vx, vy, vz, q.w, dx, dy, dz, p.tool);
            }
            if (__syncthreads_or(hit)) { found = 1; break; }
        }
        if (threadIdx.x == 0 && found) atomicOr(p.gam + i * p.grid.W + (j >> 5), 1u << (j & 31));
    }
}

// ---------------------------------------------------------------- upload helpers

__device__ __forceinline__ unsigned int float_to_ordered(float f) {
    const unsigned int u = __float_as_uint(f);
    return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ float ordered_to_float(unsigned int u) {
    return __uint_as_float((u & 0x80000000u) ? (u & 0x7fffffffu) : ~u);
}

// Validate, pack to float4 and take the bounding box (ordered-int atomics).
__global__ void pack_validate_kernel(const float* __restrict__ c, const float* __restrict__ h,
                                     long long N, float4* __restrict__ out, unsigned int* bbox,
                                     unsigned long long* bad) {
    unsigned int lo[3] = {0xffffffffu, 0xffffffffu, 0xffffffffu}, hi[3] = {0u, 0u, 0u};
    unsigned long long nbad = 0;
    for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < N;
         k += (long long)gridDim.x * blockDim.x) {
        const float x = c[3 * k], y = c[3 * k + 1], z = c[3 * k + 2], s = h[k];
        const bool ok = isfinite(x) && isfinite(y) && isfinite(z) && isfinite(s) && s > 0.f;
        nbad += !ok;
        out[k] = make_float4(x, y, z, s);
        if (ok) {
            const unsigned int o[3] = {float_to_ordered(x), float_to_ordered(y), float_to_ordered(z)};
#pragma unroll
            for (int a = 0; a < 3; ++a) {
                lo[a] = min(lo[a], o[a]);
                hi[a] = max(hi[a], o[a]);
            }
        }
    }
#pragma unroll
    for (int a = 0; a < 3; ++a) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            lo[a] = min(lo[a], __shfl_xor_sync(0xffffffffu, lo[a], o));
            hi[a] = max(hi[a], __shfl_xor_sync(0xffffffffu, hi[a], o));
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) nbad += __shfl_xor_sync(0xffffffffu, nbad, o);
    if ((threadIdx.x & 31) == 0) {
#pragma unroll
        for (int a = 0; a < 3; ++a) {
            atomicMin(bbox + a, lo[a]);
            atomicMax(bbox + 3 + a, hi[a]);
        }
        if (nbad) atomicAdd(bad, nbad);
    }
}

__device__ __forceinline__ unsigned long long spread3(unsigned int v) {
    unsigned long long x = v & 0x1fffffu;
    x = (x | x << 32) & 0x1f00000000ffffULL;
    x = (x | x << 16) & 0x1f0000ff0000ffULL;
    x = (x | x << 8) & 0x100f00f00f00f00fULL;
    x = (x | x << 4) & 0x10c30c30c30c30c3ULL;
    x = (x | x << 2) & 0x1249249249249249ULL;
    return x;
}

__global__ void morton_keys_kernel(const float4* __restrict__ v, long long N, const unsigned int* bbox,
                                   unsigned long long* keys, unsigned int* ids) {
    const float lx = ordered_to_float(bbox[0]), ly = ordered_to_float(bbox[1]), lz = ordered_to_float(bbox[2]);
    const float hx = ordered_to_float(bbox[3]), hy = ordered_to_float(bbox[4]), hz = ordered_to_float(bbox[5]);
    const float ext = fmaxf(fmaxf(hx - lx, hy - ly), fmaxf(hz - lz, 1e-30f));
    const float sc = 2097151.f / ext;
    for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < N;
         k += (long long)gridDim.x * blockDim.x) {
        const float4 q = v[k];
        const unsigned int qx = (unsigned int)fminf(fmaxf((q.x - lx) * sc, 0.f), 2097151.f);
        const unsigned int qy = (unsigned int)fminf(fmaxf((q.y - ly) * sc, 0.f), 2097151.f);
        const unsigned int qz = (unsigned int)fminf(fmaxf((q.z - lz) * sc, 0.f), 2097151.f);
        keys[k] = spread3(qx) | spread3(qy) << 1 | spread3(qz) << 2;
        ids[k] = (unsigned int)k;
    }
}

// Sort keys for the coarse levels: half-size bits (positive floats order as uints).
__global__ void size_keys_kernel(const float4* __restrict__ v, long long N, unsigned int* keys,
                                 unsigned int* ids) {
    for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < N;
         k += (long long)gridDim.x * blockDim.x) {
        keys[k] = __float_as_uint(v[k].w);
        ids[k] = (unsigned int)k;
    }
}

__global__ void strided_ids_kernel(unsigned int* ids, long long count, long long stride) {
    for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < count;
         k += (long long)gridDim.x * blockDim.x)
        ids[k] = (unsigned int)(k * stride);
}

__global__ void gather_kernel(const float4* __restrict__ src, const unsigned int* __restrict__ ids,
                              long long N, float4* __restrict__ dst) {
    for (long long k = blockIdx.x * (long long)blockDim.x + threadIdx.x; k < N;
         k += (long long)gridDim.x * blockDim.x)
        dst[k] = src[ids[k]];
}

// Packed AM (m x W words) <-> one byte per cell (m x n), for the voxel-sharded
// multi-GPU combine (all_reduce MAX over bytes is OR; over packed words it is not).
__global__ void unpack_cells_kernel(const uint32_t* __restrict__ words, GridDev g, uint8_t* __restrict__ cells) {
    const int nc = g.m * g.n;
    for (int c = blockIdx.x * blockDim.x + threadIdx.x; c < nc; c += gridDim.x * blockDim.x) {
        const int i = c / g.n, j = c - i * g.n;
        cells[c] = (uint8_t)((words[i * g.W + (j >> 5)] >> (j & 31)) & 1u);
    }
}

__global__ void pack_cells_kernel(const uint8_t* __restrict__ cells, GridDev g, uint32_t* __restrict__ words) {
    const int nw = g.m * g.W;
    for (int w = blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += gridDim.x * blockDim.x) {
        const int i = w / g.W, j0 = (w - i * g.W) << 5;
        uint32_t v = 0u;
        for (int b = 0; b < 32 && j0 + b < g.n; ++b) v |= (cells[i * g.n + j0 + b] ? 1u : 0u) << b;
        words[w] = v;
    }
}

}  // namespace am
