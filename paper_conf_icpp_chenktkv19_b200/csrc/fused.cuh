// fused.cuh -- the whole AICA map as ONE persistent cooperative kernel.
//
// The multi-kernel pipeline (stream.cuh) is a chain of ~15 dependent launches
// whose work is small and latency-bound once the clear-direction map and the
// brick culling have removed >98 % of the voxels; every launch boundary costs
// a drain, a launch and a ramp.  am_pipeline_kernel runs the same phases in
// one launch of SMs x occupancy CTAs (all co-resident: cooperative launch),
// separated by grid-wide barriers:
//
//   1. level-0 cones   (largest voxels, inner cones)      -> records/tasks
//   2. level-0 rows    (one task per thread, shared AM)    -> global AM
//   3. clear-direction map from the global AM (every CTA compacts the clear
//      cells into shared memory; one texel per thread)
//   4. level-1 voxels  (filter + inner cones, optional)    -> records/tasks
//   5. level-1 rows                                         -> global AM
//   6. clear-direction map again
//   7. brick test      (one brick per thread)               -> kept-brick list
//   8. brick voxels    (filter; the few live voxels compute both cones at once)
//   9. rows            (outer/inner/ring intervals, band pairs queued)
//  10. band            (exact CHECKBOX where the bit is still clear)
//
// Every phase uses the same device functions as the multi-kernel path, so the
// two produce the same map bit for bit (tests).
//
// Batched pivots: one map is a chain of ~10 short,
// latency-bound phases, so a single map leaves most of the GPU idle between
// barriers.  am_pipeline_kernel<true> splits the co-resident CTAs into one
// group per pivot; each group runs the same phases for its pivot, with its own
// barrier and its own slot of every per-map buffer, so K maps share the GPU
// and the barrier latency of one.
#pragma once
#include <cooperative_groups.h>

#include <type_traits>

#include "stream.cuh"

namespace am {

constexpr int kMaxSlots = 16;  // pivots per batched launch

struct FusedParams {
    StreamParams main;        // full stream: vox, bricks, cmap (written in phase 3/6), stage-2 counters
    StreamParams lvl;         // clear-map levels: scratch stats, stage-0 counters, vox = level-0 array
    const float4* l1;         // level-1 voxels (vox_coarse + n_l0, model order) and their count
    const float4* l1subs;     // bounding spheres of every 32 consecutive level-1 voxels (nullptr: not used)
    unsigned long long* clear1;  // batched: clear cells after level 0 (slot 0's word; slot-shifted), or nullptr
    int l1_sparse;            // batched: level 1 every 2nd voxel when at most this many cells are clear (0 = off)
    unsigned int n0, n1;
    unsigned int* rec1;       // stage-1 counters
    unsigned long long* task1;
    unsigned int* live1;      // level-1 live count (unused: level 1 computes cones inline)
    const float4* texels;     // clear-map texels
    const float4* texels1;    // texels of the map after level 0 when level 1 follows (cmapT1 <= main.cmapT)
    int cmapT1;
    int ntex;
    int use_l1;
    int small;                // am_latency_kernel: level 0 is the whole model, no maps / bricks (latency.cuh)
    unsigned long long* ts;   // diagnostics: %globaltimer after each phase (CTA 0), or nullptr
    // batched launch (am_pipeline_kernel<true>): the CTAs form nslot groups; group s
    // owns slot s of every per-map buffer (the slot-0 pointers above advanced by
    // s strides, in bytes) and takes pivots from a queue until it is empty.
    int nslot;
    unsigned long long ctr_stride, q_stride, rec_stride, task_stride, live_stride, cmap_stride, blist_stride;
    const float4* piv;        // npiv pivots: xyz, w = may_cull
    unsigned int npiv;
    uint32_t* gam0;           // map of pivot k at gam0 + k * m * W
    // batched path (batch.cuh): the call's output base is read from device memory (*out_ptr, written
    // with the pivots), so a captured launch chain does not depend on the caller's buffer; the maps
    // of this launch start out_off words after it.  nullptr: gam0.
    const unsigned long long* out_ptr;
    unsigned long long out_off;
    // AM_OPT_REUSE (batched path): per slot two witness arrays of m n voxel ids at wit0 + (2 slot +
    // parity) m n (a call writes parity q -- read with the output base, word 2 of *out_ptr -- and
    // reads 1 - q) and a hash set of hash_words ids (power of 2) that dedupes the witnesses it reads.
    unsigned int* wit0;
    unsigned int* hash0;
    unsigned int hash_words;
    unsigned long long* ctr0; // slot s's counters: ctr0 + s * ctr_stride bytes, ctr_words 64-bit words
    int ctr_words;
    unsigned int* qnext;      // pivot queue head (zeroed)
    unsigned int* cur;        // per group: its current pivot
    unsigned long long* bar;  // per group: [arrivals, generation] (zeroed)
};

template <typename T>
__device__ __forceinline__ T* shift_bytes(T* p, unsigned long long b) {
    return p ? reinterpret_cast<T*>(reinterpret_cast<char*>(const_cast<typename std::remove_const<T>::type*>(p)) + b)
             : p;
}

// The slot-s copy of a StreamParams: per-map buffers of slot s (the pivot and
// its map are set per pivot).
__device__ void slot_params(StreamParams& p, const FusedParams& F, int s, bool own_cmap) {
    const unsigned long long c = s * F.ctr_stride;
    p.qcount = shift_bytes(p.qcount, c);
    p.stats = shift_bytes(p.stats, c);
    p.early = shift_bytes(p.early, c);
    p.live_count = shift_bytes(p.live_count, c);
    p.rec_count = shift_bytes(p.rec_count, c);
    p.task_count = shift_bytes(p.task_count, c);
    p.brick_count = shift_bytes(p.brick_count, c);
    p.queue = shift_bytes(p.queue, s * F.q_stride);
    p.live_idx = shift_bytes(p.live_idx, s * F.live_stride);
    p.recs = shift_bytes(p.recs, s * F.rec_stride);
    p.tasks = shift_bytes(p.tasks, s * F.task_stride);
    p.brick_list = shift_bytes(p.brick_list, s * F.blist_stride);
    p.super_list = shift_bytes(p.super_list, s * F.blist_stride);
    p.super_count = shift_bytes(p.super_count, c);
    if (own_cmap) p.cmap = shift_bytes(p.cmap, s * F.cmap_stride);
}

__device__ __forceinline__ void set_pivot(StreamParams& p, float4 v, uint32_t* gam) {
    p.px = v.x;
    p.py = v.y;
    p.pz = v.z;
    p.may_cull = v.w != 0.f;
    p.gam = gam;
}

// Barrier over the nb CTAs of one group (all co-resident: cooperative launch).
// bar[0] counts arrivals, bar[1] is the generation; the last arrival resets the
// count and advances the generation.
__device__ __forceinline__ void group_sync(unsigned long long* bar, unsigned int nb) {
    __syncthreads();
    if (threadIdx.x == 0) {
        volatile unsigned long long* gen = bar + 1;
        const unsigned long long g0 = *gen;
        __threadfence();
        if (atomicAdd(bar, 1ull) == nb - 1) {
            atomicExch(bar, 0ull);
            __threadfence();
            atomicAdd(bar + 1, 1ull);
        } else {
            while (*gen == g0) __nanosleep(20);
        }
        __threadfence();
    }
    __syncthreads();
}

__device__ __forceinline__ void fused_mark(const FusedParams& F, int k) {
    if (F.ts && blockIdx.x == 0 && threadIdx.x == 0) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        F.ts[k] = t;
    }
}

// Dynamic shared memory: AM, row-full bits, then (16-byte aligned) the
// clear directions of the clear-direction map phases.
__host__ __device__ inline size_t fused_dirs_offset(int m, int W) {
    return ((size_t)(m * W + ((m + 31) >> 5) + 1) * sizeof(uint32_t) + 15) & ~(size_t)15;
}
// then the row starts of the live phase's clear list (m + 1 ints)
__host__ __device__ inline size_t fused_rows_offset(int m, int W) {
    return fused_dirs_offset(m, W) + (size_t)kMapDirs * sizeof(float4);
}
__host__ __device__ inline size_t fused_smem_bytes(int m, int W) {
    return fused_rows_offset(m, W) + (size_t)(m + 1) * sizeof(int);
}

// Seed the shared AM from the global AM and compute the row-full bits.
__device__ void fused_seed(const StreamParams& p, uint32_t* sAM, uint32_t* sRowFull) {
    const int m = p.grid.m, W = p.grid.W, MW = m * W;
    for (int w = threadIdx.x; w < MW; w += blockDim.x) sAM[w] = ld_cg(p.gam + w);
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int base = 0; base < m; base += blockDim.x) {
        const int i = base + threadIdx.x;
        bool full = false;
        if (i < m) {
            full = true;
            for (int w = 0; w < W; ++w)
                if (sAM[i * W + w] != row_word_mask(w, p.grid.n)) full = false;
        }
        const uint32_t bal = __ballot_sync(0xffffffffu, full);
        if (lane == 0 && base + warp * 32 < m) sRowFull[(base + warp * 32) >> 5] = bal;
    }
    __syncthreads();
}

// OR the shared AM into the global AM (words with new bits only).
__device__ void fused_flush(const StreamParams& p, const uint32_t* sAM) {
    __syncthreads();
    const int MW = p.grid.m * p.grid.W;
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        const uint32_t sv = sAM[w];
        if (sv & ~ld_cg(p.gam + w)) atomicOr(p.gam + w, sv);
    }
}

// Rasterise the tasks of one stage (grid-stride), into the shared AM.
template <bool COARSE>
__device__ void fused_rows(const StreamParams& p, const unsigned long long* task_count, uint32_t* sAM,
                           const uint32_t* sRowFull, Counters cnt, unsigned int gb, unsigned int gn) {
    const unsigned long long ntask = min(*reinterpret_cast<const volatile unsigned long long*>(task_count), p.task_cap);
    unsigned int rows = 0, rfull = 0;
    for (unsigned long long k = gb * (unsigned long long)blockDim.x + threadIdx.x; k < ntask;
         k += (unsigned long long)gn * blockDim.x) {
        const unsigned long long t = p.tasks[k];
        if (t == kInertTask) continue;  // (a cone rasterised inline: see emit_cones)
        const ConeRec r = p.recs[t >> 16];
        if (r.i0 < 0) continue;
        const int i = r.i0 + (int)(t & 0xffffu);
        if ((sRowFull[i >> 5] >> (i & 31)) & 1u) {
            ++rfull;
            continue;
        }
        ++rows;
        raster_row<COARSE>(p, r, i, sAM, cnt);
    }
    if (rows && cnt.c) atomicAdd(cnt.c + CT_ROWS, rows);
    if (rfull && cnt.c) atomicAdd(cnt.c + CT_ROWFULL, rfull);
}

// CTA-wide reservation (every thread of the CTA calls it): `cnt` slots for
// this thread in an array filled through the global counter `g`, with ONE
// atomic per CTA (many warps hitting one counter serialise in L2).  Returns
// this thread's first slot.  sScan: kWarps + 1 words of shared memory.
template <typename T>
__device__ __forceinline__ T cta_reserve(T cnt, T* g, T* sScan) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    T incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const T t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    if (lane == 31) sScan[warp] = incl;
    __syncthreads();
    if (threadIdx.x == 0) {
        T run = 0;
        for (int w = 0; w < kWarps; ++w) {
            const T t = sScan[w];
            sScan[w] = run;
            run += t;
        }
        sScan[kWarps] = run ? atomicAdd(g, run) : (T)0;
    }
    __syncthreads();
    const T base = sScan[kWarps] + sScan[warp] + incl - cnt;
    __syncthreads();
    return base;
}

struct FusedScratch {
    unsigned int r32[kWarps + 1];
    unsigned long long r64[kWarps + 1];
};

// Brick phase (the paper's octree pruning, Alg. 2
// L218-219, as bounding spheres over the Morton order), one brick of 256
// voxels per thread of the CTA step starting at brick b0: a brick whose sphere
// may still reach a clear cell is kept (counted in the high word of the brick
// counter, for am_stats) and its 8 sub-bricks of 32 voxels are tested the same
// way, warp-cooperatively (4 kept bricks x 8 sub-bricks per pass); the kept
// sub-bricks are appended to brick_list (count in the low word).  Without
// sub-brick spheres (AM_OPT_SUBBRICKS = 0) every sub-brick of a kept brick is
// kept.  Exact-safe: a voxel's cube lies inside each enclosing sphere.
__device__ __forceinline__ bool node_dropped(const StreamParams& P, const float4* __restrict__ spheres, unsigned int k) {
    if (!spheres) return false;
    const float4 s = __ldg(spheres + k);
    return sphere_dropped(P, s.x - P.px, s.y - P.py, s.z - P.pz, s.w);
}

__device__ __forceinline__ void brick_test(const StreamParams& P, unsigned int b, bool valid) {
    __shared__ unsigned int sKept[kWarps][32];  // per warp: its kept bricks
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const unsigned int lt = (1u << lane) - 1u;
    const unsigned long long nsub = ((unsigned long long)P.N + 31) >> 5;
    const bool kb = valid && b < P.nbricks && !node_dropped(P, P.bricks, b);
    const unsigned int mb = __ballot_sync(0xffffffffu, kb);
    if (!mb) return;
    if (lane == 0) atomicAdd(P.brick_count + 1, (unsigned int)__popc(mb));
    if (kb) sKept[warp][__popc(mb & lt)] = b;
    __syncwarp();
    const int n = __popc(mb);
    for (int u = 0; u < n; u += 4) {  // 4 kept bricks x 8 sub-bricks per pass
        const int j = u + (lane >> 3);
        const unsigned int sb = j < n ? sKept[warp][j] * 8u + (lane & 7) : 0u;
        const bool sk = j < n && sb < nsub && !node_dropped(P, P.subs, sb);
        const unsigned int mk = __ballot_sync(0xffffffffu, sk);
        if (mk) {
            unsigned int base = 0;
            if (lane == 0) base = atomicAdd(P.brick_count, (unsigned int)__popc(mk));
            base = __shfl_sync(0xffffffffu, base, 0);
            if (sk) P.brick_list[base + __popc(mk & lt)] = sb;
        }
    }
    __syncwarp();
}

__device__ __forceinline__ void brick_step(const StreamParams& P, unsigned int b0) {
    brick_test(P, b0 + threadIdx.x, true);
}

// Voxel phase, one CTA step over the kept sub-bricks [k0, k0 + kVPT kWarps):
// warp w reads sub-bricks k0 + k kWarps + w (k < kVPT), one voxel per lane (a
// coalesced 512-byte read each), through fast_filter; live voxels are appended
// to the live list with one reservation per CTA step (CTA-uniform call).
__device__ __forceinline__ void voxel_step(const StreamParams& P, unsigned int k0, unsigned int nk,
                                           FusedScratch& sc, unsigned int& nculled, unsigned int& npassed,
                                           unsigned int& streamed) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    float4 q[kVPT];
    unsigned int idx[kVPT];
    bool ok[kVPT];
#pragma unroll
    for (int k = 0; k < kVPT; ++k) {
        const unsigned int e = k0 + k * kWarps + warp;
        ok[k] = e < nk;
        idx[k] = ok[k] ? P.brick_list[e] * 32u + lane : 0u;
        ok[k] = ok[k] && idx[k] < (unsigned long long)P.N;
        q[k] = ok[k] ? __ldcs(P.vox + idx[k]) : make_float4(0.f, 0.f, 0.f, 1.f);
    }
    bool live[kVPT];
    unsigned int nl = 0;
#pragma unroll
    for (int k = 0; k < kVPT; ++k) {
        const int f = ok[k] ? fast_filter(P, q[k], P.gam) : F_DROP;
        nculled += f >> 1;
        streamed += ok[k];
        live[k] = f == F_LIVE;
        nl += live[k];
    }
    npassed += nl;
    unsigned int pos = cta_reserve<unsigned int>(nl, P.live_count, sc.r32);
#pragma unroll
    for (int k = 0; k < kVPT; ++k)
        if (live[k]) {
            if (pos < P.live_cap) P.live_idx[pos] = idx[k];  // (past it: live_overflow_rescan)
            ++pos;
        }
}

// Rows i0 .. i0 + nrows - 1 that are not yet full, word w of the row-full bits.
__device__ __forceinline__ uint32_t open_rows_word(const uint32_t* rowfull, int i0, int i1, int w) {
    uint32_t b = ~rowfull[w];
    if (w == (i0 >> 5)) b &= 0xffffffffu << (i0 & 31);
    if (w == (i1 >> 5)) b &= 0xffffffffu >> (31 - (i1 & 31));
    return b;
}

// cta_reserve of two counters at once (one scan, one barrier sequence).
__device__ __forceinline__ void cta_reserve2(unsigned int ca, unsigned int* ga, unsigned long long cb,
                                             unsigned long long* gb_, FusedScratch* sc, unsigned int& ba,
                                             unsigned long long& bb) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    unsigned int ia = ca;
    unsigned long long ib = cb;
    if (__all_sync(0xffffffffu, ca <= 1u && cb < (1ull << 20))) {
        // the common case (a record flag and a row count per thread): one 32-bit scan of
        // (ca << 25) | cb -- over 32 lanes the sums stay below 2^6 and 2^25
        unsigned int v = (ca << 25) | (unsigned int)cb;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned int t = __shfl_up_sync(0xffffffffu, v, o);
            if (lane >= o) v += t;
        }
        ia = v >> 25;
        ib = v & ((1u << 25) - 1u);
    } else {
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned int ta = __shfl_up_sync(0xffffffffu, ia, o);
            const unsigned long long tb = __shfl_up_sync(0xffffffffu, ib, o);
            if (lane >= o) {
                ia += ta;
                ib += tb;
            }
        }
    }
    if (lane == 31) {
        sc->r32[warp] = ia;
        sc->r64[warp] = ib;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned int ra = 0;
        unsigned long long rb = 0;
        for (int w = 0; w < kWarps; ++w) {
            const unsigned int ta = sc->r32[w];
            const unsigned long long tb = sc->r64[w];
            sc->r32[w] = ra;
            sc->r64[w] = rb;
            ra += ta;
            rb += tb;
        }
        sc->r32[kWarps] = ra ? atomicAdd(ga, ra) : 0u;
        sc->r64[kWarps] = rb ? atomicAdd(gb_, rb) : 0ull;
    }
    __syncthreads();
    ba = sc->r32[kWarps] + sc->r32[warp] + ia - ca;
    bb = sc->r64[kWarps] + sc->r64[warp] + ib - cb;
    __syncthreads();
}

// CTA-wide emit_cones: records at slot_off + [reserved], tasks at
// task_off + [reserved] for the rows of the cone not yet full; rows
// rasterised inline when the buffers are full.
template <bool COARSE>
__device__ __forceinline__ void emit_cones_cta(const StreamParams& p, unsigned int* rec_count,
                                               unsigned long long* task_count, unsigned int slot_off,
                                               unsigned long long task_off, unsigned int slot_cap,
                                               unsigned long long task_cap, int nrows, const ConeRec& r, bool counted,
                                               FusedScratch* sc, unsigned long long* stats,
                                               const uint32_t* rowfull) {
    const int i0 = r.i0, i1 = r.i0 + nrows - 1;
    int ntask = 0;
    if (nrows > 0)
        for (int w = i0 >> 5; w <= (i1 >> 5); ++w) ntask += __popc(open_rows_word(rowfull, i0, i1, w));
    if (stats) {  // the full stream's am_stats: live voxels, rows of their cones already full (a5)
        const unsigned int c = __popc(__ballot_sync(0xffffffffu, counted));
        const unsigned int f = __reduce_add_sync(0xffffffffu, (unsigned int)(nrows > 0 ? nrows - ntask : 0));
        if ((threadIdx.x & 31) == 0) {
            if (c) atomicAdd(stats + ST_LIVE, (unsigned long long)c);
            if (f) atomicAdd(stats + ST_ROWFULL, (unsigned long long)f);
        }
    }
    if (!__syncthreads_or(ntask > 0)) return;  // nothing to emit in the whole CTA (CTA-uniform)
    unsigned int slot;
    unsigned long long t0;
    cta_reserve2(ntask > 0 ? 1u : 0u, rec_count, (unsigned long long)ntask, task_count, sc, slot, t0);
    slot += slot_off;
    t0 += task_off;
    if (ntask > 0) {
        if (slot < slot_cap && t0 + ntask <= task_cap) {
            p.recs[slot] = r;
            unsigned long long t = t0;
            for (int w = i0 >> 5; w <= (i1 >> 5); ++w) {
                uint32_t b = open_rows_word(rowfull, i0, i1, w);
                while (b) {
                    const int i = (w << 5) + __ffs(b) - 1;
                    b &= b - 1u;
                    p.tasks[t++] = ((unsigned long long)slot << 16) | (unsigned int)(i - i0);
                }
            }
        } else {
            // buffers full: rasterise inline, and make the task entries reserved for this cone that lie
            // inside the task buffer inert (the row pass reads every entry below the capacity)
            for (int k = 0; k < nrows; ++k) raster_row<COARSE>(p, r, r.i0 + k, p.gam, Counters{nullptr});
            if (slot < slot_cap) p.recs[slot].i0 = -1;
            for (unsigned long long t = t0; t < t0 + ntask && t < task_cap; ++t) p.tasks[t] = kInertTask;
        }
    }
}

// The live list of a batched map slot holds live_cap entries (AM_OPT_LIVE_CAP); when the filter found
// more (count > cap) the ones past it were not stored.  Then the CTAs gb = 0 .. gn-1 of the live-cone
// phase send the kept sub-bricks' voxels through the same filter again and emit the cones of every live
// one -- the first cap of them a second time, which only repeats work (the map is an OR of per-voxel
// rows) -- so the map is exact.  CTA-uniform call; counts the overflow once (am_stats.queue_overflow).
__device__ void live_overflow_rescan(const StreamParams& P, unsigned int count, unsigned int gb, unsigned int gn,
                                     const float4* sDirs, int nclear, const int* sRowStart, FusedScratch* sc,
                                     const uint32_t* sRowFull) {
    if (gb == 0 && threadIdx.x == 0) atomicAdd(P.stats + ST_OVERFLOW, (unsigned long long)(count - P.live_cap));
    const unsigned int nk = *reinterpret_cast<const volatile unsigned int*>(P.brick_count);  // kept sub-bricks
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (unsigned int k0 = gb * kWarps; k0 < nk; k0 += gn * kWarps) {  // CTA-uniform; a warp per sub-brick
        const unsigned int e = k0 + warp;
        const unsigned int idx = e < nk ? P.brick_list[e] * 32u + lane : 0u;
        int nrows = 0;
        bool counted = false;
        ConeRec r;
        if (e < nk && idx < (unsigned long long)P.N) {
            const float4 q = P.vox[idx];
            if (fast_filter(P, q, P.gam) == F_LIVE)
                nrows = cone_of_voxel<false>(P, q, idx, r, counted, sDirs, nclear, 0, sRowStart);
        }
        emit_cones_cta<false>(P, P.rec_count, P.task_count, 0u, 0ull, P.rec_cap, P.task_cap, nrows, r, counted, sc,
                              P.stats, sRowFull);
    }
}

struct FusedShared {
    unsigned int cnt[CT_COUNT];
    unsigned int culled, passed, streamed;
    FusedScratch sc;
    int n;
};

// The phases of one map (P: main stream, L: clear-map levels) by the CTAs
// gb = 0..gn-1 of a group; gsync() = the group's barrier.
template <bool BATCH, typename Sync>
__device__ __forceinline__ void map_phases(const FusedParams& F, const StreamParams& P, const StreamParams& L,
                                           unsigned int* rec1, unsigned long long* task1, unsigned int gb,
                                           unsigned int gn, Sync gsync, FusedShared& S, unsigned char* smem_raw) {
    auto& sCnt = S.cnt;
    auto& sc = S.sc;
    const int m = P.grid.m, MW = m * P.grid.W;
    uint32_t* sAM = reinterpret_cast<uint32_t*>(smem_raw);
    uint32_t* sRowFull = sAM + MW;
    float4* sDirs = reinterpret_cast<float4*>(smem_raw + fused_dirs_offset(m, P.grid.W));
    const unsigned long long gstride = (unsigned long long)gn * blockDim.x;
    if (threadIdx.x < CT_COUNT) sCnt[threadIdx.x] = 0u;
    if (threadIdx.x == 0) {
        S.culled = S.passed = 0u;
        S.streamed = 0u;
    }
    const Counters none{nullptr};
    for (int w = threadIdx.x; w < ((m + 31) >> 5); w += blockDim.x) sRowFull[w] = 0u;
    __syncthreads();

    // 1. level-0 cones (inner), every voxel of the level is live (CTA-uniform loop)
    for (unsigned long long b0 = gb * (unsigned long long)blockDim.x; b0 < F.n0; b0 += gstride) {
        const unsigned long long e = b0 + threadIdx.x;
        int nrows = 0;
        bool counted = false;
        ConeRec r;
        if (e < F.n0) nrows = cone_of_voxel<true>(L, L.vox[e], (unsigned int)e, r, counted);
        emit_cones_cta<true>(L, L.rec_count, L.task_count, 0u, 0ull, L.rec_cap, L.task_cap, nrows, r, counted, &sc,
                             nullptr, sRowFull);
    }
    gsync();
    if (!BATCH || gb == 0) fused_mark(F, 1);
    // 2. level-0 rows
    for (int w = threadIdx.x; w < MW; w += blockDim.x) sAM[w] = 0u;
    for (int w = threadIdx.x; w < ((m + 31) >> 5); w += blockDim.x) sRowFull[w] = 0u;
    __syncthreads();
    fused_rows<true>(L, L.task_count, sAM, sRowFull, none, gb, gn);
    fused_flush(L, sAM);
    gsync();
    if (!BATCH || gb == 0) fused_mark(F, 2);
    // 3. clear-direction map (at cmapT1 texels per face when level 1 follows: it only filters level 1)
    //    Every CTA counts the clear cells of the same (barrier-stable) map: a full map ends the
    //    phases in all CTAs alike (early exit, a7)
    bool full = clear_map_cta(P.gam, P.grid, P.tab, F.use_l1 ? F.texels1 : F.texels, F.use_l1 ? F.cmapT1 : P.cmapT,
                              const_cast<float4*>(P.cmap), sAM, sDirs, &S.n, gb, gn) == 0;
    gsync();
    if (!BATCH || gb == 0) fused_mark(F, 3);
    if (F.use_l1 && !full) {
        // 4. level-1 voxels: filter against the map, inner cones (stage 1: upper
        //    halves of the record / task buffers; the records index the level-1 array)
        fused_seed(P, sAM, sRowFull);
        for (unsigned long long b0 = gb * (unsigned long long)blockDim.x; b0 < F.n1; b0 += gstride) {
            const unsigned long long e = b0 + threadIdx.x;
            int nrows = 0;
            bool counted = false;
            ConeRec r;
            if (e < F.n1) {
                const float4 q = F.l1[e];
                if (fast_filter(P, q, P.gam, F.cmapT1, F.texels1) == F_LIVE)
                    nrows = cone_of_voxel<true>(P, q, (unsigned int)e, r, counted, nullptr, -1, F.cmapT1, nullptr, F.texels1);
            }
            emit_cones_cta<true>(P, rec1, task1, P.rec_cap / 2, P.task_cap / 2, P.rec_cap, P.task_cap, nrows, r,
                                 counted, &sc, nullptr, sRowFull);
        }
        gsync();
        if (!BATCH || gb == 0) fused_mark(F, 4);
        // 5. level-1 rows (tasks in the upper halves)
        fused_seed(P, sAM, sRowFull);
        {
            const unsigned long long ntask =
                min(*reinterpret_cast<const volatile unsigned long long*>(task1), P.task_cap / 2);
            for (unsigned long long k = gb * (unsigned long long)blockDim.x + threadIdx.x; k < ntask;
                 k += gstride) {
                const unsigned long long t = P.tasks[P.task_cap / 2 + k];
                if (t == kInertTask) continue;
                const ConeRec r = P.recs[t >> 16];
                if (r.i0 < 0) continue;
                const int i = r.i0 + (int)(t & 0xffffu);
                if ((sRowFull[i >> 5] >> (i & 31)) & 1u) continue;
                raster_row<true>(P, r, i, sAM, none);
            }
        }
        fused_flush(P, sAM);
        gsync();
        if (!BATCH || gb == 0) fused_mark(F, 5);
        // 6. clear-direction map again
        full = clear_map_cta(P.gam, P.grid, P.tab, F.texels, P.cmapT, const_cast<float4*>(P.cmap), sAM, sDirs, &S.n,
                             gb, gn) == 0;
        gsync();
        if (!BATCH || gb == 0) fused_mark(F, 6);
    }
    if (full) {  // early exit: the coarse levels filled the map, no voxel can change it
        if (gb == 0 && threadIdx.x == 0) *P.early = 1ull;
        return;
    }
    // 7. brick test (kept bricks -> kept 32-voxel sub-bricks)
    for (unsigned int b0 = gb * kThreads; b0 < P.nbricks; b0 += gn * kThreads) brick_step(P, b0);
    gsync();
    if (!BATCH || gb == 0) fused_mark(F, 7);
    // 8a. kept sub-bricks: filter (kVPT x kWarps sub-bricks per CTA step); live voxels go
    //     to the global live list with one atomic per CTA step
    {
        unsigned int nculled = 0, npassed = 0, streamed = 0;
        const unsigned int nk = *reinterpret_cast<const volatile unsigned int*>(P.brick_count);
        for (unsigned int k0 = gb * (kVPT * kWarps); k0 < nk; k0 += gn * (kVPT * kWarps))
            voxel_step(P, k0, nk, sc, nculled, npassed, streamed);
        // warp sums, one shared atomic per warp (a 64-bit shared atomic would be a CAS loop)
        npassed = __reduce_add_sync(0xffffffffu, npassed);
        nculled = __reduce_add_sync(0xffffffffu, nculled);
        const unsigned int nstream = __reduce_add_sync(0xffffffffu, (unsigned int)streamed);
        if ((threadIdx.x & 31) == 0) {
            if (npassed) atomicAdd(&S.passed, npassed);
            if (nculled) atomicAdd(&S.culled, nculled);
            if (nstream) atomicAdd(&S.streamed, nstream);
        }
    }
    fused_seed(P, sAM, sRowFull);  // row-full bits of the global AM (unchanged until phase 9)
    gsync();
    if (!BATCH || gb == 0) fused_mark(F, 10);
    // 8b. both cones of the live voxels, spread over every thread of the grid (stage 2),
    //     checked against the list of cells still clear
    {
        int* sRowStart = reinterpret_cast<int*>(smem_raw + fused_rows_offset(m, P.grid.W));
        const int nclear = clear_list_rows_cta(sAM, P.grid, P.tab, sDirs, sRowStart);
        const unsigned int count = *reinterpret_cast<const volatile unsigned int*>(P.live_count);  // (uniform)
        const unsigned long long nlive = min(count, P.live_cap);
        for (unsigned long long b0 = gb * (unsigned long long)blockDim.x; b0 < nlive; b0 += gstride) {
            const unsigned long long e = b0 + threadIdx.x;
            int nrows = 0;
            bool counted = false;
            ConeRec r;
            if (e < nlive) {
                const unsigned int vidx = P.live_idx[e];
                nrows = cone_of_voxel<false>(P, P.vox[vidx], vidx, r, counted, sDirs, nclear, 0, sRowStart);
            }
            emit_cones_cta<false>(P, P.rec_count, P.task_count, 0u, 0ull, P.rec_cap, P.task_cap, nrows, r, counted,
                                  &sc, P.stats, sRowFull);
        }
        if (count > P.live_cap) live_overflow_rescan(P, count, gb, gn, sDirs, nclear, sRowStart, &sc, sRowFull);
    }
    gsync();
    if (!BATCH || gb == 0) fused_mark(F, 8);
    // 9. rows of the full stream (both cones, band pairs queued)
    fused_seed(P, sAM, sRowFull);
    fused_rows<false>(P, P.task_count, sAM, sRowFull, Counters{sCnt}, gb, gn);
    fused_flush(P, sAM);
    gsync();
    if (!BATCH || gb == 0) fused_mark(F, 9);
    // 10. band: exact test where the bit is still clear
    {
        const unsigned long long cntq = *reinterpret_cast<const volatile unsigned long long*>(P.qcount);
        const unsigned long long n = cntq < (unsigned long long)P.qcap ? cntq : (unsigned long long)P.qcap;
        unsigned long long tests = 0, hits = 0;
        for (unsigned long long k = gb * (unsigned long long)blockDim.x + threadIdx.x; k < n; k += gstride) {
            const unsigned long long e = P.queue[k];
            const unsigned int vidx = (unsigned int)(e >> 32);
            const int cell = (int)(e & 0xffffffffu);
            const int i = cell / P.grid.n, j = cell - i * P.grid.n;
            uint32_t* wp = P.gam + i * P.grid.W + (j >> 5);
            const uint32_t bit = 1u << (j & 31);
            if (ld_cg(wp) & bit) continue;
            ++tests;
            if (exact_pair(P, P.vox_main[vidx], cell)) {
                ++hits;
                atomicOr(wp, bit);
            }
        }
        if (tests) atomicAdd(P.stats + ST_EXACT, tests);
        if (hits) atomicAdd(P.stats + ST_EXACT_HIT, hits);
    }
    __syncthreads();
    if (!BATCH) fused_mark(F, 15);
    if (threadIdx.x == 0) {
        atomicAdd(P.stats + ST_CULLED, (unsigned long long)S.culled);
        atomicAdd(P.stats + ST_PASSED, (unsigned long long)S.passed);
        atomicAdd(P.stats + ST_STREAMED, (unsigned long long)S.streamed);
        atomicAdd(P.stats + ST_ROWS, (unsigned long long)sCnt[CT_ROWS]);
        atomicAdd(P.stats + ST_BAND, (unsigned long long)sCnt[CT_BAND]);
        atomicAdd(P.stats + ST_OVERFLOW, (unsigned long long)sCnt[CT_OVERFLOW]);
        atomicAdd(P.stats + ST_ROWFULL, (unsigned long long)sCnt[CT_ROWFULL]);
    }
}


// BATCH = false: one map, the whole grid, cooperative-groups grid barriers.
// BATCH = true: F.nslot groups of contiguous CTAs; each group takes pivots from
// the queue F.qnext until it is empty and computes their maps with its own
// slot of the per-map buffers and its own barrier (a slow pivot delays only
// its group).
template <bool BATCH>
__global__ void __launch_bounds__(kThreads, 2) am_pipeline_kernel(const __grid_constant__ FusedParams F) {
    namespace cg = cooperative_groups;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ FusedShared S;
    if (!BATCH) {
        fused_mark(F, 0);
        map_phases<false>(F, F.main, F.lvl, F.rec1, F.task1, blockIdx.x, gridDim.x,
                          []() { cg::this_grid().sync(); }, S, smem_raw);
        return;
    }
    __shared__ StreamParams sP, sL;
    __shared__ unsigned int* sRec1;
    __shared__ unsigned long long* sTask1;
    // group of this CTA: CTAs [start(s), start(s + 1)), start(s) = s * G / nslot
    const unsigned int G = gridDim.x;
    const unsigned int K = (unsigned int)F.nslot;
    const unsigned int slot = (unsigned int)(((blockIdx.x + 1ull) * K - 1ull) / G);
    const unsigned int gstart = (unsigned int)((unsigned long long)slot * G / K);
    const unsigned int gb = blockIdx.x - gstart;
    const unsigned int gn = (unsigned int)((unsigned long long)(slot + 1) * G / K) - gstart;
    unsigned long long* bar = F.bar + 2 * slot;
    unsigned long long* ctr = shift_bytes(F.ctr0, slot * F.ctr_stride);
    fused_mark(F, 0);
    if (threadIdx.x == 0) {
        sP = F.main;
        sL = F.lvl;
        slot_params(sP, F, (int)slot, true);
        slot_params(sL, F, (int)slot, false);
        sRec1 = shift_bytes(F.rec1, slot * F.ctr_stride);
        sTask1 = shift_bytes(F.task1, slot * F.ctr_stride);
    }
    auto gsync = [bar, gn]() { group_sync(bar, gn); };
    const int MW = F.main.grid.m * F.main.grid.W;
    while (true) {
        if (gb == 0 && threadIdx.x == 0) F.cur[slot] = atomicAdd(F.qnext, 1u);
        group_sync(bar, gn);
        const unsigned int k = *reinterpret_cast<volatile unsigned int*>(F.cur + slot);
        if (k >= F.npiv) break;
        uint32_t* gam = F.gam0 + (size_t)k * MW;
        if (threadIdx.x == 0) {
            const float4 v = F.piv[k];
            set_pivot(sP, v, gam);
            set_pivot(sL, v, gam);
        }
        if (gb == 0) {  // this pivot's map and the slot's counters start at zero
            for (int w = threadIdx.x; w < MW; w += blockDim.x) gam[w] = 0u;
            for (int w = threadIdx.x; w < F.ctr_words; w += blockDim.x) ctr[w] = 0ull;
        }
        group_sync(bar, gn);
        map_phases<true>(F, sP, sL, sRec1, sTask1, gb, gn, gsync, S, smem_raw);
    }
}

}  // namespace am
