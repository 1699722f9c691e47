// stage.cuh -- the batched path's stages as one kernel each (AM_OPT_STAGE_FUSION; default off).
//
// The batched chain (batch.cuh) splits each stage in a cone kernel that writes cone records and
// (cone, phi-row) tasks to global memory and a row kernel that reads them back; the live stage is
// a third kernel before them (the voxel filter).  Here each stage is ONE launch per chunk of
// pivots (blockIdx.y = pivot, as in batch.cuh), built from the single-pivot kernel's CTA-local
// pieces (latency.cuh): filters buffer their survivors in shared memory, the survivors' cones wait
// in shared memory and every (cone, row) pair is a task for the whole CTA (cta_raster), then the
// CTA's shared AM is OR-ed into the map.  No record/task round trip through HBM, two launches and
// two prologues fewer per chunk.  Work is dealt to the CTAs of a pivot round robin (element e to
// CTA e mod gridDim.x), so the survivors -- a spatially clustered few of each Morton-ordered array
// -- spread over every CTA.
//
//   bk_level0  level 0 + (AM_OPT_REUSE) the previous map's witnesses: inner cones, rows
//   bk_level1  level 1: filter against the first map, inner cones, rows
//   bk_stream  the kept sub-bricks' voxels: filter -> both cones -> exact outer cone vs the CTA's
//              clear list -> rows -> band pairs queued   (replaces bk_voxels, bk_cones<LIVE>,
//              bk_rows<LIVE>)
//
// The per-(voxel, cell) decisions are those of the split kernels (same device functions), so the
// maps are bit-identical (tests).  Measured on B200 (C3, 64 maps per step): 10.8 us per map against
// 6.4 with the split kernels -- with 64 maps in flight the split kernels' global task lists keep
// every thread busy, while a CTA-local drain leaves most threads idle during the cones (one thread
// per survivor) and the fused stages need more registers (3 CTAs per SM).  So the option is off by
// default; the same pieces make the single-pivot kernel fast (latency.cuh), where the GPU idles.
#pragma once
#include "batch.cuh"
#include "latency.cuh"

#ifndef AM_STAGE_MIN_BLOCKS
#define AM_STAGE_MIN_BLOCKS 3
#endif
// the coarse levels (inner cones only, no clear list: launched with the AM + row-full bits as their
// only dynamic shared memory) fit more CTAs per SM
#ifndef AM_STAGE_LEVEL_MIN_BLOCKS
#define AM_STAGE_LEVEL_MIN_BLOCKS 5
#endif

namespace am {

struct StageSmem {
    uint32_t* sAM;
    uint32_t* sRowFull;
    float4* sDirs;
    int* sRowStart;
};

__device__ __forceinline__ StageSmem stage_smem(unsigned char* raw, int m, int W) {
    StageSmem s;
    s.sAM = reinterpret_cast<uint32_t*>(raw);
    s.sRowFull = s.sAM + m * W;
    s.sDirs = reinterpret_cast<float4*>(raw + fused_dirs_offset(m, W));
    s.sRowStart = reinterpret_cast<int*>(raw + fused_rows_offset(m, W));
    return s;
}

__device__ __forceinline__ void stage_init(LatShared& S) {
    if (threadIdx.x < CT_COUNT) S.cnt[threadIdx.x] = 0u;
    if (threadIdx.x == 0) {
        S.culled = S.passed = S.streamed = S.live = 0u;
        S.nl = 0;
    }
    __syncthreads();
}

// Level 0 (+ the reuse witnesses) of pivot blockIdx.y: inner cones, rows, straight to the map.
__global__ void __launch_bounds__(kThreads, AM_STAGE_LEVEL_MIN_BLOCKS) bk_level0(const __grid_constant__ FusedParams F) {
    extern __shared__ __align__(16) unsigned char smem_st[];
    __shared__ StreamParams sP;
    __shared__ LatShared S;
    const int p = blockIdx.y;
    pivot_params(sP, F, p, true);
    const StreamParams& P = sP;
    const StageSmem sm = stage_smem(smem_st, P.grid.m, P.grid.W);
    stage_init(S);
    const unsigned int* prev = nullptr;  // AM_OPT_REUSE: the previous map's witnesses of this slot
    unsigned int* hs = nullptr;
    unsigned long long n = F.n0;
    if (F.wit0) {
        const unsigned int mn = (unsigned int)(P.grid.m * P.grid.n);
        prev = F.wit0 + (2ull * p + (1u - reuse_parity(F))) * mn;
        hs = F.hash0 + (unsigned long long)p * F.hash_words;
        n += mn;
    }
    lat_clear(sm.sAM, sm.sRowFull, P.grid.m, P.grid.m * P.grid.W);  // (the map is still empty: bk_init)
    unsigned int scratch = 0;
    const unsigned long long G = gridDim.x, stride = G * blockDim.x;
    for (unsigned long long c0 = 0; c0 < n; c0 += stride) {  // CTA-uniform; element e to CTA e mod G
        const unsigned long long e = c0 + (unsigned long long)threadIdx.x * G + blockIdx.x;
        ConeRec r;
        bool counted = false;
        int nrows = 0;
        if (e < n) {
            unsigned int id = e < F.n0 ? (0x80000000u | (unsigned int)e) : prev[e - F.n0];
            if (e >= F.n0 && (id == kNoWitness || !hash_insert(hs, F.hash_words, id))) id = kNoWitness;
            if (id != kNoWitness) {
                const float4 q = (id & 0x80000000u) ? P.vox_coarse[id & 0x7fffffffu] : P.vox_main[id];
                nrows = cone_of_voxel<true>(P, q, id, r, counted);
            }
        }
        cta_raster<true>(P, r, nrows, sm.sAM, sm.sRowFull, Counters{nullptr}, S, scratch, scratch);
    }
    fused_flush(P, sm.sAM);
}

// Level 1 of pivot blockIdx.y: filter against the map after level 0, inner cones, rows.
__global__ void __launch_bounds__(kThreads, AM_STAGE_LEVEL_MIN_BLOCKS) bk_level1(const __grid_constant__ FusedParams F) {
    extern __shared__ __align__(16) unsigned char smem_st[];
    __shared__ StreamParams sP;
    __shared__ LatShared S;
    const int p = blockIdx.y;
    pivot_params(sP, F, p, false);
    const StreamParams& P = sP;
    if (map_full(P.early)) return;
    const StageSmem sm = stage_smem(smem_st, P.grid.m, P.grid.W);
    stage_init(S);
    fused_seed(P, sm.sAM, sm.sRowFull);
    unsigned int scratch = 0;
    int buffered = 0;
    const unsigned long long G = gridDim.x, stride = G * blockDim.x;
    for (unsigned long long c0 = 0; c0 < F.n1; c0 += stride) {  // CTA-uniform
        const unsigned long long e = c0 + (unsigned long long)threadIdx.x * G + blockIdx.x;
        bool keep = false;
        if (e < F.n1) {
            const float4 q = F.l1[e];
            keep = fast_filter(P, q, P.gam, F.cmapT1, F.texels1) == F_LIVE;
            if (keep) lat_keep(S, q, 0x80000000u | (F.n0 + (unsigned int)e));
        }
        buffered += __syncthreads_count(keep);
        if (buffered > kLiveBuf - (int)blockDim.x) {
            lat_drain<true>(P, sm.sAM, sm.sRowFull, Counters{nullptr}, S, scratch, scratch, scratch, nullptr, -1,
                            nullptr, F.cmapT1, F.texels1);
            buffered = 0;
        }
    }
    lat_drain<true>(P, sm.sAM, sm.sRowFull, Counters{nullptr}, S, scratch, scratch, scratch, nullptr, -1, nullptr,
                    F.cmapT1, F.texels1);
    fused_flush(P, sm.sAM);
}

// The kept sub-bricks' voxels of pivot blockIdx.y: filter, both cones, rows, band queue.
__global__ void __launch_bounds__(kThreads, AM_STAGE_MIN_BLOCKS) bk_stream(const __grid_constant__ FusedParams F) {
    extern __shared__ __align__(16) unsigned char smem_st[];
    __shared__ StreamParams sP;
    __shared__ LatShared S;
    const int p = blockIdx.y;
    pivot_params(sP, F, p, false);
    const StreamParams& P = sP;
    const unsigned int nk = *reinterpret_cast<const volatile unsigned int*>(P.brick_count);
    if (blockIdx.x >= nk) return;  // CTA-uniform: no sub-brick for this CTA (it would take blockIdx.x first)
    if (map_full(P.early)) return;
    const StageSmem sm = stage_smem(smem_st, P.grid.m, P.grid.W);
    stage_init(S);
    fused_seed(P, sm.sAM, sm.sRowFull);
    const int nclear = clear_list_rows_cta(sm.sAM, P.grid, P.tab, sm.sDirs, sm.sRowStart);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    unsigned int rows = 0, rfull = 0, nlive = 0;
    int buffered = 0;
    const unsigned int G = gridDim.x;
    for (unsigned int e0 = 0; e0 < nk; e0 += G * kWarps) {  // CTA-uniform; warp w: sub-brick e0 + w G + CTA
        const unsigned int e = e0 + warp * G + blockIdx.x;
        const unsigned int sb = e < nk ? P.brick_list[e] : 0u;
        const unsigned int idx = sb * 32u + lane;
        const bool ok = e < nk && idx < (unsigned long long)P.N;
        const float4 q = ok ? __ldcs(P.vox + idx) : make_float4(0.f, 0.f, 0.f, 1.f);
        const int f = ok ? fast_filter(P, q, P.gam) : F_DROP;
        if (f == F_LIVE) lat_keep(S, q, idx);
        buffered += __syncthreads_count(f == F_LIVE);
        if (buffered > kLiveBuf - (int)blockDim.x) {
            lat_drain<false>(P, sm.sAM, sm.sRowFull, Counters{S.cnt}, S, rows, rfull, nlive, sm.sDirs, nclear,
                             sm.sRowStart, 0, nullptr);
            buffered = 0;
        }
    }
    lat_drain<false>(P, sm.sAM, sm.sRowFull, Counters{S.cnt}, S, rows, rfull, nlive, sm.sDirs, nclear, sm.sRowStart, 0,
                     nullptr);
    fused_flush(P, sm.sAM);
}

}  // namespace am
