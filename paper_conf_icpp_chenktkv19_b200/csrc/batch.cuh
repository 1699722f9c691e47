// batch.cuh -- the AICA maps of a batch of pivots, one launch per phase.
//
// The fused kernel (fused.cuh) minimises the latency of ONE map, but a map is
// a chain of ~10 short phases whose work is a few hundred thousand voxels: one
// map keeps the GPU busy only in bursts, and the fused kernel's register
// budget (the heaviest phase sets it for all) caps occupancy at 16 warps/SM.
// For a toolpath batch the same phases run here as
// separate kernels over a chunk of pivots at once: blockIdx.y is the pivot,
// each pivot owns slot blockIdx.y of every per-map buffer (the slot-0 pointers
// of FusedParams advanced by the slot strides; am.cu shifts them per stream
// lane), and each kernel gets the registers -- and so the occupancy -- its
// own phase needs.  Kernel boundaries replace the grid barriers, and the
// block scheduler balances pivots of different cost.  The host runs the
// chunks on several streams and replays the whole chain as a CUDA graph.
//
// Phases (same device functions as fused.cuh, so the maps are bit-identical):
//   bk_cones<L0>  level-0 inner cones        -> stage-0 records/tasks
//   bk_rows<0>    their rows                 -> map
//   bk_map        clear-direction map
//   bk_cones<L1>  level-1 filter + cones     -> stage-1 records/tasks
//   bk_rows<1>, bk_map
//   bk_supers     super-brick test           -> kept super-bricks
//   bk_bricks     their bricks, then the kept bricks' sub-bricks -> kept sub-bricks
//   bk_voxels     kept sub-bricks' voxels filter -> live list
//   bk_cones<LIVE> both cones of live voxels -> stage-2 records/tasks
//   bk_rows<2>    rows + band queue
//   bk_band       exact test of queued band pairs still clear
#pragma once
#include "fused.cuh"

// CTAs per SM each stage is compiled for (register budget vs occupancy)
#ifndef AM_LIVE_MIN_BLOCKS
#define AM_LIVE_MIN_BLOCKS 5
#endif
#ifndef AM_LEVEL_ROWS_MIN_BLOCKS
#define AM_LEVEL_ROWS_MIN_BLOCKS 8
#endif
#ifndef AM_MAP1_WARP_TEXEL
#define AM_MAP1_WARP_TEXEL 0  // the map after level 0: one warp per texel (1) or 8x8 texel blocks (0)
#endif
#ifndef AM_MAP_MIN_BLOCKS
#define AM_MAP_MIN_BLOCKS 5  // (48 registers; 6 and 8 measured slower, profiles/r5_sweeps.txt)
#endif
#ifndef AM_LEVEL_CONES_MIN_BLOCKS
#define AM_LEVEL_CONES_MIN_BLOCKS 8
#endif

namespace am {

// Start of this launch's maps: the call's output base (device memory, written with the pivots) or gam0.
__device__ __forceinline__ uint32_t* launch_maps(const FusedParams& F) {
    return F.out_ptr ? reinterpret_cast<uint32_t*>(*reinterpret_cast<const volatile unsigned long long*>(F.out_ptr)) +
                           F.out_off
                     : F.gam0;
}

// Programmatic dependent launch (AM_OPT_PDL): the batched kernels of a lane are launched with
// programmatic stream serialisation, so a kernel's CTAs are scheduled while the previous kernel's
// last CTAs still run and do their parameter prologue meanwhile; before touching anything the
// previous kernels wrote (counts, maps, lists) every thread waits here for them to complete and
// their writes to be visible.  A no-op for a kernel launched without the attribute.  Every CTA of a
// batched kernel passes it (also on its early-exit paths), so a kernel completes only after its
// predecessor did -- the dependency stays transitive along the lane.
__device__ __forceinline__ void grid_dep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

constexpr unsigned int kNoWitness = 0xffffffffu;

// Insert id into the open-addressing set hs (nwords a power of 2, empty = kNoWitness): true when it
// was not there yet (the caller then owns the id).
__device__ __forceinline__ bool hash_insert(unsigned int* hs, unsigned int nwords, unsigned int id) {
    unsigned int h = (id * 2654435761u) & (nwords - 1u);
    for (unsigned int k = 0; k < nwords; ++k) {
        const unsigned int old = atomicCAS(hs + h, kNoWitness, id);
        if (old == kNoWitness) return true;
        if (old == id) return false;
        h = (h + 1u) & (nwords - 1u);
    }
    return true;  // (full: process it anyway)
}

// AM_OPT_REUSE: the parity of this call (word 2 of the output-base entry written with the pivots).
__device__ __forceinline__ unsigned int reuse_parity(const FusedParams& F) {
    return reinterpret_cast<const volatile unsigned int*>(F.out_ptr)[2] & 1u;
}

// StreamParams of pivot p (slot p) into shared memory (thread 0; the kernel
// parameter is read by plain member access: a dynamically indexed pointer into
// a __grid_constant__ parameter is not a global address); `lvl` selects the
// clear-map-level copy.  Ends with a barrier.
__device__ __forceinline__ void pivot_params(StreamParams& out, const FusedParams& F, int p, bool lvl) {
    // the copy one word per thread (a ~1 KB struct copied by one thread is a long
    // serial chain in every CTA's prologue), then thread 0 applies slot and pivot
    constexpr int kWords = (int)(sizeof(StreamParams) / 4);
    uint32_t* dst = reinterpret_cast<uint32_t*>(&out);
    if (lvl) {
        const uint32_t* src = reinterpret_cast<const uint32_t*>(&F.lvl);
        for (int w = threadIdx.x; w < kWords; w += blockDim.x) dst[w] = src[w];
    } else {
        const uint32_t* src = reinterpret_cast<const uint32_t*>(&F.main);
        for (int w = threadIdx.x; w < kWords; w += blockDim.x) dst[w] = src[w];
    }
    grid_dep_wait();
    __syncthreads();
    if (threadIdx.x == 0) {
        slot_params(out, F, p, !lvl);
        set_pivot(out, F.piv[p], launch_maps(F) + (size_t)p * F.main.grid.m * F.main.grid.W);
        if (F.wit0)  // AM_OPT_REUSE: this map's witnesses (parity q)
            out.wit = F.wit0 + (2ull * p + reuse_parity(F)) * (out.grid.m * out.grid.n);
    }
    __syncthreads();
}

// The prologue of a batched kernel (every thread calls it; ends CTA-uniformly): pivot_params plus
// the phase's work count and the early-exit check, with every device-memory read the CTA needs --
// pivot, output base, reuse parity, the count `cnt` (32- or 64-bit, slot-shifted by the caller from
// the kernel parameters) and the map's early-exit flag -- issued by thread 0 BEFORE the parameter
// copy, so their latency overlaps it (pivot_params reads them after its first barrier, and every
// kernel read its count and the flag after pivot_params).  Returns true when the CTA has nothing to
// do: the map is full (check_early; a7) or its first item `first` lies at or past the count;
// n = min(count, cap).
__device__ __forceinline__ bool bk_prologue(StreamParams& out, const FusedParams& F, int p, bool lvl, const void* cnt,
                                            bool wide, unsigned long long cap, unsigned long long first,
                                            bool check_early, unsigned long long& n) {
    __shared__ unsigned long long s_n;
    __shared__ int s_exit;
    constexpr int kWords = (int)(sizeof(StreamParams) / 4);
    float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
    unsigned long long ob = 0ull;
    unsigned int par = 0u;
    if (threadIdx.x == 0) {  // (the call's inputs: written before the lane's first kernel)
        v = F.piv[p];
        if (F.out_ptr) {
            ob = *reinterpret_cast<const volatile unsigned long long*>(F.out_ptr);
            if (F.wit0) par = reinterpret_cast<const volatile unsigned int*>(F.out_ptr)[2] & 1u;
        }
    }
    uint32_t* dst = reinterpret_cast<uint32_t*>(&out);
    if (lvl) {
        const uint32_t* src = reinterpret_cast<const uint32_t*>(&F.lvl);
        for (int w = threadIdx.x; w < kWords; w += blockDim.x) dst[w] = src[w];
    } else {
        const uint32_t* src = reinterpret_cast<const uint32_t*>(&F.main);
        for (int w = threadIdx.x; w < kWords; w += blockDim.x) dst[w] = src[w];
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        slot_params(out, F, p, !lvl);
        uint32_t* base = F.out_ptr ? reinterpret_cast<uint32_t*>(ob) + F.out_off : F.gam0;
        set_pivot(out, v, base + (size_t)p * F.main.grid.m * F.main.grid.W);
        if (F.wit0) out.wit = F.wit0 + (2ull * p + par) * (out.grid.m * out.grid.n);
    }
    grid_dep_wait();  // (everything below reads what the previous kernels wrote)
    if (threadIdx.x == 0) {
        unsigned long long c = ~0ull;
        if (cnt)
            c = wide ? *reinterpret_cast<const volatile unsigned long long*>(cnt)
                     : (unsigned long long)*reinterpret_cast<const volatile unsigned int*>(cnt);
        const bool full =
            check_early &&
            *reinterpret_cast<const volatile unsigned long long*>(shift_bytes(F.main.early, p * F.ctr_stride)) != 0ull;
        const unsigned long long nn = c < cap ? c : cap;
        s_n = nn;
        s_exit = full || first >= nn;
    }
    __syncthreads();
    n = s_n;
    return s_exit != 0;  // (CTA-uniform)
}

// First launch of a chunk: zero the maps and the per-slot counters of its pivots (blockIdx.x = pivot).
__global__ void __launch_bounds__(kThreads) bk_init(const __grid_constant__ FusedParams F) {
    grid_dep_wait();
    const int p = blockIdx.x;
    const int MW = F.main.grid.m * F.main.grid.W;
    uint32_t* g = launch_maps(F) + (size_t)p * MW;
    for (int w = threadIdx.x; w < MW; w += blockDim.x) g[w] = 0u;
    unsigned long long* c = shift_bytes(F.ctr0, p * F.ctr_stride);
    for (int w = threadIdx.x; w < F.ctr_words; w += blockDim.x) c[w] = 0ull;
    if (F.wit0) {  // (AM_OPT_REUSE) no witness yet; an empty dedupe set
        const int mn = F.main.grid.m * F.main.grid.n;
        unsigned int* wit = F.wit0 + (2ull * p + reuse_parity(F)) * mn;
        for (int w = threadIdx.x; w < mn; w += blockDim.x) wit[w] = kNoWitness;
        unsigned int* hs = F.hash0 + (unsigned long long)p * F.hash_words;
        for (unsigned int w = threadIdx.x; w < F.hash_words; w += blockDim.x) hs[w] = kNoWitness;
    }
}

enum { BK_L0 = 0, BK_L1 = 1, BK_LIVE = 2 };

// Cones of one stage: level 0 (every voxel of the level, inner cones), level 1
// (filtered against the map, inner cones), or the live voxels (both cones).
template <int STAGE>
__global__ void __launch_bounds__(kThreads, STAGE == 2 ? AM_LIVE_MIN_BLOCKS : AM_LEVEL_CONES_MIN_BLOCKS) bk_cones(const __grid_constant__ FusedParams F) {
    extern __shared__ __align__(16) uint32_t smem_bk[];
    __shared__ StreamParams sP;
    __shared__ FusedScratch sc;
    const int p = blockIdx.y;
    unsigned long long n;
    unsigned int l1s = 1;  // level 1: every l1s-th voxel (AM_OPT_L1_SPARSE)
    if constexpr (STAGE == BK_L1) {
        // (the prologue's count: the clear cells the map after level 0 left, written by bk_map<true>)
        const bool sparse = F.l1_sparse > 0 && F.clear1;
        if (bk_prologue(sP, F, p, false, sparse ? (const void*)shift_bytes(F.clear1, p * F.ctr_stride) : nullptr, true,
                        ~0ull, 0ull, true, n))
            return;
        l1s = (sparse && n <= (unsigned long long)F.l1_sparse) ? 2u : 1u;
        n = (F.n1 + l1s - 1) / l1s;
        if ((unsigned long long)blockIdx.x * blockDim.x >= n) return;  // CTA-uniform
    } else {
        const void* cnt = STAGE == BK_LIVE ? (const void*)shift_bytes(F.main.live_count, p * F.ctr_stride) : nullptr;
        const unsigned long long cap = STAGE == BK_L0 ? ~0ull : (unsigned long long)F.main.live_cap;
        if (bk_prologue(sP, F, p, STAGE == BK_L0, cnt, false, cap, (unsigned long long)blockIdx.x * blockDim.x,
                        STAGE != BK_L0, n))
            return;
    }
    const StreamParams& P = sP;
    const int m = P.grid.m, MW = m * P.grid.W;
    uint32_t* sAM = smem_bk;
    uint32_t* sRowFull = sAM + MW;
    float4* sDirs = reinterpret_cast<float4*>(reinterpret_cast<unsigned char*>(smem_bk) + fused_dirs_offset(m, P.grid.W));
    int* sRowStart = reinterpret_cast<int*>(reinterpret_cast<unsigned char*>(smem_bk) + fused_rows_offset(m, P.grid.W));
    int nclear = -1;
    const unsigned int* prev = nullptr;  // AM_OPT_REUSE: the previous map's witnesses of this slot
    unsigned int* hs = nullptr;
    if (STAGE == BK_L0) {
        n = F.n0;
        if (F.wit0) {
            const unsigned int mn = (unsigned int)(P.grid.m * P.grid.n);
            prev = F.wit0 + (2ull * p + (1u - reuse_parity(F))) * mn;
            hs = F.hash0 + (unsigned long long)p * F.hash_words;
            n += mn;
        }
        for (int w = threadIdx.x; w < ((m + 31) >> 5); w += blockDim.x) sRowFull[w] = 0u;
        __syncthreads();
    } else {
        // (n: level 1's size, or the live count read by the prologue)
        fused_seed(P, sAM, sRowFull);
        if (STAGE == BK_LIVE) nclear = clear_list_rows_cta(sAM, P.grid, P.tab, sDirs, sRowStart);
    }
    unsigned int* rc = STAGE == BK_L1 ? shift_bytes(F.rec1, p * F.ctr_stride) : P.rec_count;
    unsigned long long* tc = STAGE == BK_L1 ? shift_bytes(F.task1, p * F.ctr_stride) : P.task_count;
    const unsigned int roff = STAGE == BK_L1 ? P.rec_cap / 2 : 0u;
    const unsigned long long toff = STAGE == BK_L1 ? P.task_cap / 2 : 0ull;
    const unsigned int rcap = P.rec_cap;  // (level 0: the level copy's caps are the lower halves)
    const unsigned long long tcap = P.task_cap;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long b0 = blockIdx.x * (unsigned long long)blockDim.x; b0 < n; b0 += stride) {
        const unsigned long long e = b0 + threadIdx.x;
        int nrows = 0;
        bool counted = false;
        ConeRec r;
        if (e < n) {
            if (STAGE == BK_L0) {
                // level 0, then the previous map's witnesses (AM_OPT_REUSE), each once: their inner cones
                // at this pivot.  Ids: bit 31 = the coarse array (levels 0 and 1), else the model
                unsigned int id = e < F.n0 ? (0x80000000u | (unsigned int)e) : prev[e - F.n0];
                if (e >= F.n0 && (id == kNoWitness || !hash_insert(hs, F.hash_words, id))) id = kNoWitness;
                if (id != kNoWitness) {
                    const float4 q = (id & 0x80000000u) ? P.vox_coarse[id & 0x7fffffffu] : P.vox_main[id];
                    nrows = cone_of_voxel<true>(P, q, id, r, counted);
                }
            } else if (STAGE == BK_L1) {
                // (the warp's 32 voxels are one level-1 group: skipped together when the group's sphere
                //  cannot reach a clear cell -- b0 is a multiple of blockDim, so the warp is group-aligned)
                bool group = true;
                if (F.l1subs && l1s == 1) {
                    const float4 g = __ldg(F.l1subs + ((b0 + (threadIdx.x & ~31u)) >> 5));
                    group = !sphere_dropped(P, g.x - P.px, g.y - P.py, g.z - P.pz, g.w, F.cmapT1, F.texels1);
                }
                const unsigned long long el = e * l1s;
                const float4 q = F.l1[el];
                if (group && fast_filter(P, q, P.gam, F.cmapT1, F.texels1) == F_LIVE)
                    nrows = cone_of_voxel<true>(P, q, 0x80000000u | (F.n0 + (unsigned int)el), r, counted, nullptr, -1,
                                                F.cmapT1, nullptr, F.texels1);
            } else {
                const unsigned int vidx = P.live_idx[e];
                nrows = cone_of_voxel<false>(P, P.vox[vidx], vidx, r, counted, sDirs, nclear, 0, sRowStart);
            }
        }
        emit_cones_cta<STAGE != BK_LIVE>(P, rc, tc, roff, toff, rcap, tcap, nrows, r, counted, &sc,
                                         STAGE == BK_LIVE ? P.stats : nullptr, sRowFull);
    }
    if (STAGE == BK_LIVE) {  // the slot's live list overflowed (AM_OPT_LIVE_CAP): fused.cuh live_overflow_rescan
        __shared__ unsigned int s_count;
        if (threadIdx.x == 0) s_count = *reinterpret_cast<const volatile unsigned int*>(P.live_count);
        __syncthreads();
        const unsigned int count = s_count;
        if (count > P.live_cap) {  // (CTA-uniform) by the CTAs that did not exit for lack of list entries
            const unsigned int gn = (unsigned int)min((unsigned long long)gridDim.x, (n + blockDim.x - 1) / blockDim.x);
            live_overflow_rescan(P, count, blockIdx.x, gn, sDirs, nclear, sRowStart, &sc, sRowFull);
        }
    }
}

// Rows of one stage into the CTA's shared AM (seeded from the map, so rows
// already full are skipped), then OR-ed into the map.
template <int STAGE>
__global__ void __launch_bounds__(kThreads, STAGE == 2 ? AM_LIVE_MIN_BLOCKS : AM_LEVEL_ROWS_MIN_BLOCKS) bk_rows(const __grid_constant__ FusedParams F) {
    extern __shared__ __align__(16) uint32_t smem_bk[];
    __shared__ StreamParams sP;
    __shared__ unsigned int sCnt[CT_COUNT];
    const int p = blockIdx.y;
    if (threadIdx.x < CT_COUNT) sCnt[threadIdx.x] = 0u;
    unsigned long long ntask;
    {
        // (compile-time choices: a run-time select between two kernel-parameter addresses is not valid)
        const unsigned long long* tc;
        unsigned long long cap;
        if constexpr (STAGE == BK_L0) {
            tc = shift_bytes(F.lvl.task_count, p * F.ctr_stride);
            cap = F.lvl.task_cap;
        } else if constexpr (STAGE == BK_L1) {
            tc = shift_bytes(F.task1, p * F.ctr_stride);
            cap = F.main.task_cap / 2;
        } else {
            tc = shift_bytes(F.main.task_count, p * F.ctr_stride);
            cap = F.main.task_cap;
        }
        if (bk_prologue(sP, F, p, STAGE == BK_L0, tc, true, cap, (unsigned long long)blockIdx.x * blockDim.x,
                        STAGE != BK_L0, ntask))
            return;
    }
    const StreamParams& P = sP;
    uint32_t* sAM = smem_bk;
    uint32_t* sRowFull = sAM + P.grid.m * P.grid.W;
    fused_seed(P, sAM, sRowFull);
    const unsigned long long toff = STAGE == BK_L1 ? P.task_cap / 2 : 0ull;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned int rows = 0, rfull = 0;
    for (unsigned long long k = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; k < ntask; k += stride) {
        const unsigned long long t = P.tasks[toff + k];
        if (t == kInertTask) continue;  // (a cone rasterised inline: see emit_cones)
        const ConeRec r = P.recs[t >> 16];
        if (r.i0 < 0) continue;
        const int i = r.i0 + (int)(t & 0xffffu);
        if ((sRowFull[i >> 5] >> (i & 31)) & 1u) {
            ++rfull;
            continue;
        }
        ++rows;
        raster_row<STAGE != BK_LIVE>(P, r, i, sAM, Counters{STAGE == BK_LIVE ? sCnt : nullptr});
    }
    fused_flush(P, sAM);
    if (STAGE == BK_LIVE) {
        rows = __reduce_add_sync(0xffffffffu, rows);
        rfull = __reduce_add_sync(0xffffffffu, rfull);
        if ((threadIdx.x & 31) == 0 && rows) atomicAdd(&sCnt[CT_ROWS], rows);
        if ((threadIdx.x & 31) == 0 && rfull) atomicAdd(&sCnt[CT_ROWFULL], rfull);
        __syncthreads();
        if (threadIdx.x == 0) {
            if (sCnt[CT_ROWS]) atomicAdd(P.stats + ST_ROWS, (unsigned long long)sCnt[CT_ROWS]);
            if (sCnt[CT_BAND]) atomicAdd(P.stats + ST_BAND, (unsigned long long)sCnt[CT_BAND]);
            if (sCnt[CT_OVERFLOW]) atomicAdd(P.stats + ST_OVERFLOW, (unsigned long long)sCnt[CT_OVERFLOW]);
            if (sCnt[CT_ROWFULL]) atomicAdd(P.stats + ST_ROWFULL, (unsigned long long)sCnt[CT_ROWFULL]);
        }
    }
}

// Clear-direction map of pivot p's map (kernels.cuh clear_map_cta); FIRST: the
// map after level 0 when level 1 follows, at F.cmapT1 texels per face.
template <bool FIRST>
__global__ void __launch_bounds__(kThreads, AM_MAP_MIN_BLOCKS) bk_map(const __grid_constant__ FusedParams F) {
    extern __shared__ __align__(16) unsigned char smem_bm[];
    __shared__ StreamParams sP;
    __shared__ int sN;
    const int p = blockIdx.y;
    unsigned long long unused;
    if (bk_prologue(sP, F, p, false, nullptr, false, ~0ull, 0ull, true, unused)) return;
    const StreamParams& P = sP;
    uint32_t* sAM = reinterpret_cast<uint32_t*>(smem_bm);
    float4* sDirs = reinterpret_cast<float4*>(smem_bm + fused_dirs_offset(P.grid.m, P.grid.W));
    const int total = clear_map_cta(P.gam, P.grid, P.tab, FIRST ? F.texels1 : F.texels, FIRST ? F.cmapT1 : P.cmapT,
                                    const_cast<float4*>(P.cmap), sAM, sDirs, &sN, blockIdx.x, gridDim.x,
                                    FIRST && AM_MAP1_WARP_TEXEL, !FIRST);
    if (total == 0 && blockIdx.x == 0 && threadIdx.x == 0) *P.early = 1ull;  // early exit (a7)
    if (FIRST && F.clear1 && blockIdx.x == 0 && threadIdx.x == 0)  // (AM_OPT_L1_SPARSE: for bk_cones<L1>)
        *shift_bytes(F.clear1, p * F.ctr_stride) = (unsigned long long)total;
}

// Super-brick test (P.supers set): super-bricks of 8 bricks whose bounding
// sphere may still reach a clear cell go to the map's super list.
__global__ void __launch_bounds__(kThreads) bk_supers(const __grid_constant__ FusedParams F) {
    __shared__ StreamParams sP;
    const int p = blockIdx.y;
    unsigned long long unused;
    if (bk_prologue(sP, F, p, false, nullptr, false, ~0ull, 0ull, true, unused)) return;
    const StreamParams& P = sP;
    const int lane = threadIdx.x & 31;
    const unsigned int nsup = (P.nbricks + 7) >> 3;
    for (unsigned int s0 = blockIdx.x * kThreads; s0 < nsup; s0 += gridDim.x * kThreads) {
        const unsigned int sp = s0 + threadIdx.x;
        const bool keep = sp < nsup && !node_dropped(P, P.supers, sp);
        const unsigned int mk = __ballot_sync(0xffffffffu, keep);
        if (!mk) continue;
        unsigned int base = 0;
        if (lane == 0) base = atomicAdd(P.super_count, (unsigned int)__popc(mk));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (keep) P.super_list[base + __popc(mk & ((1u << lane) - 1u))] = sp;
    }
}

// Brick test: bricks (all, or the 8 of each kept super-brick), then their
// 32-voxel sub-bricks, whose bounding sphere may still reach a clear cell
// (fused.cuh brick_test).
__global__ void __launch_bounds__(kThreads) bk_bricks(const __grid_constant__ FusedParams F) {
    __shared__ StreamParams sP;
    const int p = blockIdx.y;
    unsigned long long unused;
    if (bk_prologue(sP, F, p, false, nullptr, false, ~0ull, 0ull, true, unused)) return;
    const StreamParams& P = sP;
    if (P.supers) {
        const unsigned int ne = 8u * *reinterpret_cast<const volatile unsigned int*>(P.super_count);
        for (unsigned int e0 = blockIdx.x * kThreads; e0 < ne; e0 += gridDim.x * kThreads) {
            const unsigned int e = e0 + threadIdx.x;
            const unsigned int b = e < ne ? P.super_list[e >> 3] * 8u + (e & 7u) : 0u;
            brick_test(P, b, e < ne);
        }
    } else {
        for (unsigned int b0 = blockIdx.x * kThreads; b0 < P.nbricks; b0 += gridDim.x * kThreads) brick_step(P, b0);
    }
}

// AM_FUSED_BRICKS: super-bricks -> their bricks -> the kept bricks' sub-bricks in ONE launch (the
// single-pivot kernel's P5): every warp tests 32 super-bricks dealt transposed over the pivot's warps (the
// kept ones, a spatially clustered few, land on different warps), then the 8 bricks of each kept one,
// 4 kept super-bricks x 8 lanes per pass (brick_test, which tests the sub-bricks of the kept bricks).
__global__ void __launch_bounds__(kThreads) bk_bricks_fused(const __grid_constant__ FusedParams F) {
    __shared__ StreamParams sP;
    __shared__ unsigned int sKeptS[kWarps][32];
    const int p = blockIdx.y;
    unsigned long long unused;
    if (bk_prologue(sP, F, p, false, nullptr, false, ~0ull, 0ull, true, unused)) return;
    const StreamParams& P = sP;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const unsigned int nsup = (P.nbricks + 7) >> 3;
    const unsigned int nw = gridDim.x * kWarps, gw = blockIdx.x * kWarps + warp;
    for (unsigned int k0 = 0; k0 < nsup; k0 += nw * 32) {  // (uniform bound)
        const unsigned int sp = k0 + lane * nw + gw;
        const bool keep = sp < nsup && !node_dropped(P, P.supers, sp);
        const unsigned int mk = __ballot_sync(0xffffffffu, keep);
        if (keep) sKeptS[warp][__popc(mk & ((1u << lane) - 1u))] = sp;
        __syncwarp();
        const int n = __popc(mk);
        for (int u = 0; u < n; u += 4) {  // 4 kept super-bricks x 8 bricks per pass
            const int j = u + (lane >> 3);
            const unsigned int b = j < n ? sKeptS[warp][j] * 8u + (lane & 7) : 0u;
            brick_test(P, b, j < n);
        }
        __syncwarp();
    }
}

// Kept sub-bricks' voxels through the filter; live voxels to the live list.
__global__ void __launch_bounds__(kThreads) bk_voxels(const __grid_constant__ FusedParams F) {
    __shared__ StreamParams sP;
    __shared__ FusedScratch sc;
    __shared__ unsigned int sStat[3];
    const int p = blockIdx.y;
    if (threadIdx.x < 3) sStat[threadIdx.x] = 0u;
    unsigned long long nk64;
    if (bk_prologue(sP, F, p, false, shift_bytes(F.main.brick_count, p * F.ctr_stride), false, ~0ull,
                    (unsigned long long)blockIdx.x * (kVPT * kWarps), true, nk64))
        return;
    const StreamParams& P = sP;
    const unsigned int nk = (unsigned int)nk64;
    unsigned int nculled = 0, npassed = 0, streamed = 0;
    for (unsigned int k0 = blockIdx.x * (kVPT * kWarps); k0 < nk; k0 += gridDim.x * (kVPT * kWarps))
        voxel_step(P, k0, nk, sc, nculled, npassed, streamed);
    npassed = __reduce_add_sync(0xffffffffu, npassed);
    nculled = __reduce_add_sync(0xffffffffu, nculled);
    streamed = __reduce_add_sync(0xffffffffu, streamed);
    if ((threadIdx.x & 31) == 0) {
        if (npassed) atomicAdd(&sStat[0], npassed);
        if (nculled) atomicAdd(&sStat[1], nculled);
        if (streamed) atomicAdd(&sStat[2], streamed);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (sStat[0]) atomicAdd(P.stats + ST_PASSED, (unsigned long long)sStat[0]);
        if (sStat[1]) atomicAdd(P.stats + ST_CULLED, (unsigned long long)sStat[1]);
        if (sStat[2]) atomicAdd(P.stats + ST_STREAMED, (unsigned long long)sStat[2]);
    }
}

// Band: exact test of the queued pairs whose bit is still clear.  Each warp checks 32 pairs (one
// per lane; lane j of warp w takes pair w + j W of the W warps of the pivot, so that the open
// pairs, neighbours in the queue, land on different warps) and runs CHECKBOX on the still-clear
// ones with the whole warp (exact_hit_warp: the sub-tests side by side, ~4x less latency than one
// thread's chain).
__global__ void __launch_bounds__(kThreads) bk_band(const __grid_constant__ FusedParams F) {
    __shared__ StreamParams sP;
    const int p = blockIdx.y;
    unsigned long long n;
    if (bk_prologue(sP, F, p, false, shift_bytes(F.main.qcount, p * F.ctr_stride), true,
                    (unsigned long long)F.main.qcap, (unsigned long long)blockIdx.x * (blockDim.x >> 5), false, n))
        return;
    const StreamParams& P = sP;
    const unsigned long long nw = (unsigned long long)gridDim.x * (blockDim.x >> 5);  // warps of this pivot
    const unsigned long long gw = (unsigned long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (gw >= n) return;  // (warp-uniform: no pair for this warp)
    const int lane = threadIdx.x & 31;
    unsigned long long tests = 0, hits = 0;
    for (unsigned long long k0 = 0; k0 < n; k0 += nw * 32) {  // warp-uniform
        const unsigned long long k = k0 + lane * nw + gw;
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
            if (P.band_vdepth > 0) {  // corner-case expansion (§4.3): one lane (exact_pair)
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
        if (tests) atomicAdd(P.stats + ST_EXACT, tests);
        if (hits) atomicAdd(P.stats + ST_EXACT_HIT, hits);
    }
}

}  // namespace am
