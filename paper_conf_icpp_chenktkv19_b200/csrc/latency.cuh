// latency.cuh -- ONE pivot's AM with the shortest critical path (am_compute; the per-rank work of
// the voxel-sharded multi-GPU mode).
//
// A single map is a chain of short, data-dependent phases; on one pivot most of the GPU idles and
// every phase costs its slowest CTA's serial chain plus a grid barrier (ncu of the previous
// single-pivot kernel: 71 % of the warp samples waited at a barrier, IPC 0.15).  This kernel keeps
// the phases of the batched path (same device functions, same per-(voxel, cell) decisions, so the
// same map bit for bit) but cuts their number and spreads each over all co-resident warps:
//
//   P1 level 0 (largest voxels): one WARP per voxel -- the lanes share the cone and take its
//      phi-rows -- rasterised into the CTA's shared AM, no record/task round trip (small models:
//      an even sample of the model, one voxel per warp)
//   P2 clear-direction map of the partial AM (few texels: one warp per texel, lanes over the clear
//      directions)
//   P3 level 1: filter against the map; the survivors' inner cones and rows (CTA raster)
//   P4 clear-direction map again (a full map ends the kernel: early exit, a7)
//   P5 super-bricks -> their bricks -> the kept bricks' 32-voxel sub-bricks, in one pass: every warp
//      tests super-bricks spread over the whole model (transposed assignment, so the kept ones -- a
//      spatially clustered few -- land on different warps), then the 8 bricks of each kept one and
//      the 8 sub-bricks of each kept brick, 4 x 8 lanes per pass
//   P6 the kept sub-bricks' voxels (one warp per sub-brick, a coalesced 512-byte read, sub-bricks
//      dealt round robin over the CTAs): filter -> live voxels buffered per CTA -> both cones ->
//      exact outer cone vs the CTA's list of cells still clear -> rows (CTA raster) -> band pairs
//   P7 band: CHECKBOX of the queued pairs still clear, one warp per test (exact_hit_warp)
//
// CTA raster: the cones of a CTA's threads wait in shared memory and every (cone, phi-row) pair is
// one task for the whole CTA -- balanced whatever the cone sizes, without a grid barrier or a
// global record/task round trip.  Filters run first and buffer their survivors per CTA, so the
// cones and rows of a phase run once, with every thread busy.
//
// Small models (N <= kSmallModel, or no coarse levels): no level 1, maps or bricks; P6 streams every
// sub-brick against the map P1's sample left (its clear list does the culling).  The map's counters
// are zeroed by CTA 0 in P1 (nothing counts before the first barrier).
#pragma once
#include <cooperative_groups.h>

#include "fused.cuh"

namespace am {

constexpr long long kSmallModel = 1ll << 16;  // voxels: up to this, no coarse levels / maps / bricks

constexpr int kLiveBuf = 512;
constexpr int kDiagCtas = 1024;  // AM_OPT_DIAG bit 2: per-CTA P6 records kept for the first CTAs  // per CTA: voxels that passed a filter, waiting for their cones

struct LatShared {
    float4 liveq[kLiveBuf];          // filter survivors of this CTA (voxel) ...
    unsigned int livei[kLiveBuf];    // ... and their index
    int nl;                          // how many
    unsigned int cnt[CT_COUNT];
    unsigned int culled, passed, streamed, live;
    unsigned int keptS[kWarps][32];  // P5: per warp, its kept super-bricks
    ConeRec rec[kThreads];           // cta_raster: one cone per thread
    int pre[kThreads + 1];           // and the prefix sums of their row counts
    int wsum[kWarps];
    int n;
};

// CTA-cooperative raster (CTA-uniform call): every thread's cone (nrows phi-rows from r.i0) is
// split into (cone, row) tasks that all threads of the CTA then share, one row each -- balanced
// whatever the cone sizes, without a grid barrier or a global record/task round trip.  The cones
// wait in shared memory (one record per thread), a CTA scan of the row counts gives each task its
// cone (binary search over the prefix sums).  Rows marked full in rowfull are skipped (rfull).
template <bool COARSE>
__device__ __forceinline__ void cta_raster(const StreamParams& p, const ConeRec& r, int nrows, uint32_t* sAM,
                                           const uint32_t* rowfull, Counters cnt, LatShared& S, unsigned int& rows,
                                           unsigned int& rfull) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (nrows > 0) S.rec[threadIdx.x] = r;
    int incl = nrows;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    if (lane == 31) S.wsum[warp] = incl;
    __syncthreads();
    if (threadIdx.x == 0) {
        int run = 0;
        for (int w = 0; w < kWarps; ++w) {
            const int t = S.wsum[w];
            S.wsum[w] = run;
            run += t;
        }
        S.pre[kThreads] = run;
    }
    __syncthreads();
    S.pre[threadIdx.x] = S.wsum[warp] + incl - nrows;  // exclusive prefix
    __syncthreads();
    const int T = S.pre[kThreads];
    for (int t = threadIdx.x; t < T; t += blockDim.x) {
        int lo = 0, hi = kThreads - 1;  // the last owner o with pre[o] <= t
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (S.pre[mid] <= t) lo = mid;
            else hi = mid - 1;
        }
        const int i = S.rec[lo].i0 + (t - S.pre[lo]);
        if ((rowfull[i >> 5] >> (i & 31)) & 1u) {
            ++rfull;
            continue;
        }
        ++rows;
        raster_row<COARSE>(p, S.rec[lo], i, sAM, cnt);
    }
    __syncthreads();  // (S.rec / S.pre are reused by the next call)
}

// Cones + rows of the CTA's buffered filter survivors (CTA-uniform call), then an empty buffer.
// COARSE: level 1 (inner cones, filtered against the map of texels tex / T); else the full
// stream's live voxels (both cones, exact outer cone vs the clear list sDirs / sRowStart).
template <bool COARSE>
__device__ __forceinline__ void lat_drain(const StreamParams& p, uint32_t* sAM, const uint32_t* rowfull,
                                          Counters cnt, LatShared& S, unsigned int& rows, unsigned int& rfull,
                                          unsigned int& nlive, const float4* sDirs, int nclear, const int* sRowStart,
                                          int T, const float4* tex) {
    __syncthreads();
    const int nl = min(S.nl, kLiveBuf);
    for (int b = 0; b < nl; b += blockDim.x) {
        const int t = b + threadIdx.x;
        ConeRec r;
        bool counted = false;
        int nrows = 0;
        if (t < nl) {
            nrows = COARSE ? cone_of_voxel<true>(p, S.liveq[t], S.livei[t], r, counted, nullptr, -1, T, nullptr, tex)
                           : cone_of_voxel<false>(p, S.liveq[t], S.livei[t], r, counted, sDirs, nclear, 0, sRowStart);
            nlive += counted;
        }
        cta_raster<COARSE>(p, r, nrows, sAM, rowfull, cnt, S, rows, rfull);
    }
    __syncthreads();
    if (threadIdx.x == 0) S.nl = 0;
    __syncthreads();
}

// Append a filter survivor to the CTA's buffer (the caller drains before it can overflow).
__device__ __forceinline__ void lat_keep(LatShared& S, float4 q, unsigned int idx) {
    const int pos = atomicAdd(&S.nl, 1);
    S.liveq[pos] = q;
    S.livei[pos] = idx;
}

// Zero the shared AM and the row-full bits (no row known full).
__device__ __forceinline__ void lat_clear(uint32_t* sAM, uint32_t* sRowFull, int m, int MW) {
    for (int w = threadIdx.x; w < MW; w += blockDim.x) sAM[w] = 0u;
    for (int w = threadIdx.x; w < ((m + 31) >> 5); w += blockDim.x) sRowFull[w] = 0u;
    __syncthreads();
}

template <typename Sync>
__device__ void lat_phases(const FusedParams& F, Sync gsync, LatShared& S, unsigned char* smem_raw) {
    const StreamParams& P = F.main;
    const StreamParams& L = F.lvl;
    const int m = P.grid.m, MW = m * P.grid.W;
    uint32_t* sAM = reinterpret_cast<uint32_t*>(smem_raw);
    uint32_t* sRowFull = sAM + MW;
    float4* sDirs = reinterpret_cast<float4*>(smem_raw + fused_dirs_offset(m, P.grid.W));
    int* sRowStart = reinterpret_cast<int*>(smem_raw + fused_rows_offset(m, P.grid.W));
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const unsigned int gb = blockIdx.x, gn = gridDim.x;
    const unsigned int nw = gn * kWarps;                  // warps of the grid
    const unsigned int gw = gb * kWarps + warp;           // this warp
    const unsigned long long gstride = (unsigned long long)gn * blockDim.x;
    const Counters none{nullptr};
    const bool small = F.small != 0;  // level 0 = the whole model, no level 1 / maps / bricks
    if (threadIdx.x < CT_COUNT) S.cnt[threadIdx.x] = 0u;
    if (threadIdx.x == 0) {
        S.culled = S.passed = S.streamed = S.live = 0u;
        S.nl = 0;
    }
    if (gb == 0)  // this map's counters start at zero (P1 uses none; the first grid barrier orders it)
        for (int w = threadIdx.x; w < F.ctr_words; w += blockDim.x) F.ctr0[w] = 0ull;
    unsigned int rows = 0, rfull = 0, scratch = 0;
    (void)scratch;

    // P1: level 0 (small model: an even sample of at most one voxel per warp), inner cones, one
    // WARP per voxel -- the lanes share its cone and take its rows -- straight into the shared AM
    lat_clear(sAM, sRowFull, m, MW);
    {
        const unsigned int stride = small ? (unsigned int)((F.n0 + nw - 1) / nw) : 1u;
        const unsigned int n0 = (F.n0 + stride - 1) / stride;
        for (unsigned int v = gw; v < n0; v += nw) {
            ConeRec r;
            bool counted;
            const int nrows = cone_of_voxel<true>(L, L.vox[v * stride], v * stride, r, counted);
            for (int k = lane; k < nrows; k += 32) raster_row<true>(L, r, r.i0 + k, sAM, none);
        }
    }
    fused_flush(L, sAM);
    gsync();
    fused_mark(F, 1);
    bool full = false;
    if (!small) {
        // P2: clear-direction map of the partial AM (at cmapT1 texels per face: it only filters level 1)
        full = clear_map_cta(P.gam, P.grid, P.tab, F.use_l1 ? F.texels1 : F.texels, F.use_l1 ? F.cmapT1 : P.cmapT,
                             const_cast<float4*>(P.cmap), sAM, sDirs, &S.n, gb, gn, true) == 0;
        gsync();
        fused_mark(F, 2);
        if (F.use_l1 && !full) {
            // P3: level 1 -- filter, inner cone, rows in one pass
            fused_seed(P, sAM, sRowFull);
            // (voxels dealt to the CTAs round robin -- CTA gb takes gb, gb + gn, ... -- so the survivors, a
            //  spatially clustered few of the Morton-ordered level, spread over every CTA's raster)
            // (filter first, survivors buffered per CTA; cones and rows once the buffer is nearly full)
            int buffered = 0;  // = S.nl, kept in a register so every thread takes the same branch
            for (unsigned long long c0 = 0; c0 < F.n1; c0 += gstride) {  // CTA-uniform
                const unsigned long long e = c0 + (unsigned long long)threadIdx.x * gn + gb;
                bool keep = false;
                if (e < F.n1) {
                    const float4 q = F.l1[e];
                    keep = fast_filter(P, q, P.gam, F.cmapT1, F.texels1) == F_LIVE;
                    if (keep) lat_keep(S, q, (unsigned int)e);
                }
                buffered += __syncthreads_count(keep);
                if (buffered > kLiveBuf - (int)blockDim.x) {
                    lat_drain<true>(P, sAM, sRowFull, none, S, scratch, scratch, scratch, nullptr, -1, nullptr,
                                    F.cmapT1, F.texels1);
                    buffered = 0;
                }
            }
            lat_drain<true>(P, sAM, sRowFull, none, S, scratch, scratch, scratch, nullptr, -1, nullptr, F.cmapT1,
                            F.texels1);
            fused_flush(P, sAM);
            gsync();
            fused_mark(F, 3);
            // P4: the map again, at full resolution
            full = clear_map_cta(P.gam, P.grid, P.tab, F.texels, P.cmapT, const_cast<float4*>(P.cmap), sAM, sDirs,
                                 &S.n, gb, gn, false, true) == 0;
            gsync();
            fused_mark(F, 4);
        }
        if (full) {  // early exit: the coarse levels filled the map (CTA-uniform: one barrier-stable map)
            if (gb == 0 && threadIdx.x == 0) *P.early = 1ull;
            return;
        }
        // P5: super-bricks -> bricks -> sub-bricks (kept sub-bricks to brick_list)
        if (P.supers) {
            const unsigned int nsup = (P.nbricks + 7) >> 3;
            for (unsigned int k0 = 0; k0 < nsup; k0 += nw * 32) {  // (uniform bound)
                const unsigned int sp = k0 + lane * nw + gw;         // transposed: a warp's lanes nw apart
                const bool keep = sp < nsup && !node_dropped(P, P.supers, sp);
                const unsigned int mk = __ballot_sync(0xffffffffu, keep);
                if (keep) S.keptS[warp][__popc(mk & ((1u << lane) - 1u))] = sp;
                __syncwarp();
                const int n = __popc(mk);
                for (int u = 0; u < n; u += 4) {  // 4 kept super-bricks x 8 bricks per pass
                    const int j = u + (lane >> 3);
                    const unsigned int b = j < n ? S.keptS[warp][j] * 8u + (lane & 7) : 0u;
                    brick_test(P, b, j < n);
                }
                __syncwarp();
            }
        } else {
            for (unsigned int b0 = gb * kThreads; b0 < P.nbricks; b0 += gn * kThreads) brick_step(P, b0);
        }
        gsync();
        fused_mark(F, 5);
    }
    // P6: voxels of the kept sub-bricks (small model: every sub-brick) -> filter -> live cones -> rows
    fused_seed(P, sAM, sRowFull);
    const int nclear = clear_list_rows_cta(sAM, P.grid, P.tab, sDirs, sRowStart);
    fused_mark(F, 7);
    if (nclear == 0) {  // (small model: level 0 filled the map) early exit, CTA-uniform
        if (gb == 0 && threadIdx.x == 0) *P.early = 1ull;
        return;
    }
    {
        const unsigned long long nsub = ((unsigned long long)P.N + 31) >> 5;
        const unsigned int nk = small ? (unsigned int)nsub : *reinterpret_cast<const volatile unsigned int*>(P.brick_count);
        unsigned int nculled = 0, npassed = 0, streamed = 0, nlive = 0;
        int buffered = 0;
        // (filter first, live voxels buffered per CTA; cones and rows once the buffer is nearly full.
        //  Sub-bricks dealt round robin -- warp w of CTA gb takes e0 + w gn + gb -- so that neighbours in
        //  the list, which are neighbours in space, land on different CTAs and the live voxels spread)
        for (unsigned int e0 = 0; e0 < nk; e0 += nw) {  // CTA-uniform
            const unsigned int e = e0 + warp * gn + gb;
            const unsigned int sb = e < nk ? (small ? e : P.brick_list[e]) : 0u;
            const unsigned int idx = sb * 32u + lane;
            const bool ok = e < nk && idx < (unsigned long long)P.N;
            const float4 q = ok ? __ldcs(P.vox + idx) : make_float4(0.f, 0.f, 0.f, 1.f);
            const int f = ok ? fast_filter(P, q, P.gam) : F_DROP;
            nculled += f >> 1;
            streamed += ok;
            if (f == F_LIVE) {
                ++npassed;
                lat_keep(S, q, idx);
            }
            buffered += __syncthreads_count(f == F_LIVE);
            if (buffered > kLiveBuf - (int)blockDim.x) {
                lat_drain<false>(P, sAM, sRowFull, Counters{S.cnt}, S, rows, rfull, nlive, sDirs, nclear, sRowStart, 0,
                                 nullptr);
                buffered = 0;
            }
        }
        fused_mark(F, 8);
        lat_drain<false>(P, sAM, sRowFull, Counters{S.cnt}, S, rows, rfull, nlive, sDirs, nclear, sRowStart, 0,
                         nullptr);
        fused_mark(F, 9);
        npassed = __reduce_add_sync(0xffffffffu, npassed);
        nculled = __reduce_add_sync(0xffffffffu, nculled);
        streamed = __reduce_add_sync(0xffffffffu, streamed);
        nlive = __reduce_add_sync(0xffffffffu, nlive);
        if (lane == 0) {
            if (npassed) atomicAdd(&S.passed, npassed);
            if (nculled) atomicAdd(&S.culled, nculled);
            if (streamed) atomicAdd(&S.streamed, streamed);
            if (nlive) atomicAdd(&S.live, nlive);
        }
    }
    rows = __reduce_add_sync(0xffffffffu, rows);
    rfull = __reduce_add_sync(0xffffffffu, rfull);
    if (lane == 0) {
        if (rows) atomicAdd(&S.cnt[CT_ROWS], rows);
        if (rfull) atomicAdd(&S.cnt[CT_ROWFULL], rfull);
    }
    fused_flush(P, sAM);
    if (F.ts && threadIdx.x == 0 && gb < kDiagCtas) {  // diagnostics: this CTA's P6 end, live voxels, rows
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        F.ts[16 + 4 * gb] = t;
        F.ts[16 + 4 * gb + 1] = S.live;
        F.ts[16 + 4 * gb + 2] = S.cnt[CT_ROWS];
        F.ts[16 + 4 * gb + 3] = S.passed;
    }
    gsync();
    fused_mark(F, 6);
    // P7: band -- the exact test of the queued pairs still clear: each warp checks 32 pairs (one per
    // lane; lane j of warp w takes pair w + j nw, so that the open pairs -- neighbours in the queue,
    // pushed by one row -- land on different warps), then runs CHECKBOX on the still-clear ones one
    // after the other with the whole warp (exact_hit_warp: its sub-tests side by side)
    {
        const unsigned long long cntq = *reinterpret_cast<const volatile unsigned long long*>(P.qcount);
        const unsigned long long n = cntq < (unsigned long long)P.qcap ? cntq : (unsigned long long)P.qcap;
        unsigned int tests = 0, hits = 0;
        for (unsigned long long k0 = 0; k0 < n; k0 += (unsigned long long)nw * 32) {  // (uniform)
            const unsigned long long k = k0 + (unsigned long long)lane * nw + gw;
            unsigned long long e = 0;
            bool open = false;
            if (k < n) {
                e = P.queue[k];
                const int cell = (int)(e & 0xffffffffu);
                const int i = cell / P.grid.n, j = cell - i * P.grid.n;
                open = !(ld_cg(P.gam + i * P.grid.W + (j >> 5)) & (1u << (j & 31)));
            }
            unsigned int mo = __ballot_sync(0xffffffffu, open);
            while (mo) {
                const int src = __ffs(mo) - 1;
                mo &= mo - 1u;
                const unsigned long long es = __shfl_sync(0xffffffffu, e, src);
                const unsigned int vidx = (unsigned int)(es >> 32);
                const int cell = (int)(es & 0xffffffffu);
                const int i = cell / P.grid.n, j = cell - i * P.grid.n;
                uint32_t* wp = P.gam + i * P.grid.W + (j >> 5);
                const uint32_t bit = 1u << (j & 31);
                if (ld_cg(wp) & bit) continue;  // (blocked meanwhile; warp-uniform)
                ++tests;
                const float4 q = P.vox_main[vidx];
                bool hit;
                if (P.band_vdepth > 0) {
                    hit = __shfl_sync(0xffffffffu, lane == 0 && exact_pair(P, q, cell), 0);
                } else {
                    const float* t = P.tab;
                    const float cph = __ldg(t + i), sph = __ldg(t + P.grid.m + i);
                    const float cg = __ldg(t + 2 * P.grid.m + j), sg = __ldg(t + 2 * P.grid.m + P.grid.n + j);
                    hit = exact_hit_warp(q.x - P.px, q.y - P.py, q.z - P.pz, q.w, sph * cg, sph * sg, cph, P.tool);
                }
                if (hit) {
                    ++hits;
                    if (lane == 0) atomicOr(wp, bit);
                }
            }
        }
        if (lane == 0) {
            if (tests) atomicAdd(P.stats + ST_EXACT, (unsigned long long)tests);
            if (hits) atomicAdd(P.stats + ST_EXACT_HIT, (unsigned long long)hits);
        }
    }
    __syncthreads();
    fused_mark(F, 15);
    if (threadIdx.x == 0) {
        if (S.culled) atomicAdd(P.stats + ST_CULLED, (unsigned long long)S.culled);
        if (S.passed) atomicAdd(P.stats + ST_PASSED, (unsigned long long)S.passed);
        if (S.streamed) atomicAdd(P.stats + ST_STREAMED, (unsigned long long)S.streamed);
        if (S.live) atomicAdd(P.stats + ST_LIVE, (unsigned long long)S.live);
        if (S.cnt[CT_ROWS]) atomicAdd(P.stats + ST_ROWS, (unsigned long long)S.cnt[CT_ROWS]);
        if (S.cnt[CT_BAND]) atomicAdd(P.stats + ST_BAND, (unsigned long long)S.cnt[CT_BAND]);
        if (S.cnt[CT_OVERFLOW]) atomicAdd(P.stats + ST_OVERFLOW, (unsigned long long)S.cnt[CT_OVERFLOW]);
        if (S.cnt[CT_ROWFULL]) atomicAdd(P.stats + ST_ROWFULL, (unsigned long long)S.cnt[CT_ROWFULL]);
    }
}

__global__ void __launch_bounds__(kThreads, 2) am_latency_kernel(const __grid_constant__ FusedParams F) {
    namespace cg = cooperative_groups;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ LatShared S;
    fused_mark(F, 0);
    if (F.ts && threadIdx.x == 0) {  // diagnostics: first / last CTA start and last CTA end
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        atomicMin(F.ts + 12, t);
        atomicMax(F.ts + 13, t);
    }
    lat_phases(F, []() { cg::this_grid().sync(); }, S, smem_raw);
    if (F.ts && threadIdx.x == 0) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        atomicMax(F.ts + 14, t);
    }
}

}  // namespace am
