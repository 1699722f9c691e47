// stream.cuh -- the voxel-streaming AICA kernels.
//
// aica_stream_kernel (the full stream, every voxel):
//   Every warp is an independent worker with its own 3-stage ring in shared
//   memory.  Lane 0 claims chunks of 128 voxels (4 chunks per atomic) and pulls
//   them global -> shared with the 1-D TMA engine (cp.async.bulk + mbarrier
//   complete_tx; SASS UBLKCP), so the HBM stream runs ahead of the arithmetic
//   without registers and without CTA-wide barriers.  Per voxel the warp runs a
//   cheap, exact-safe FILTER (fast_filter): reach cull, then the cheap outer cone
//   -- a sphere of radius sqrt(3) h at distance D only touches cylinders that
//   start within D + sqrt(3) h, of radius at most Reff, so its blocked directions
//   satisfy sin(theta) <= (Reff + sqrt3 h) / D -- against the clear-direction map
//   (kernels.cuh clear_map_kernel).  A voxel whose cheap cone holds no
//   still-clear cell cannot change the AM and is dropped.  Survivors ("live",
//   ~1-2 % at the paper's 1 mm offset) go to a per-warp queue (ballot) and are
//   processed 32 at a time, one per lane (process_live): the paper's two ICA
//   cones (Alg. 1) rasterised row by row into the CTA's shared AM,
//   band cells deferred to the global band queue.  Each warp merges the shared
//   AM with the global AM on its own (a7).
//
// coarse_kernel (levels 0/1, the largest voxels):
//   one warp per voxel, phi-rows across lanes, inner cones only -- these few
//   voxels have cones spanning most rows, so row parallelism is what they need.
#pragma once
#include "kernels.cuh"

namespace am {

constexpr int kWarps = kThreads / 32;
constexpr int kChunk = 128;     // voxels per TMA copy (4 per lane)
constexpr int kWStages = 3;     // per-warp ring depth
constexpr int kSuper = 4;       // chunks claimed per atomic
constexpr int kWQ = 64;         // per-warp live queue (drained at 32)
static_assert(sizeof(StreamParams) % 4 == 0 && sizeof(StreamParams) / 4 <= kThreads,
              "StreamParams is copied to shared memory one word per thread");

__device__ __forceinline__ unsigned int smem_u32(const void* p) {
    return static_cast<unsigned int>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned int count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, unsigned int bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned int parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

// 1-D bulk copy global -> shared, completion signalled on `bar` (bytes % 16 == 0).
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, unsigned int bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

__device__ __forceinline__ float rcp_approx(float x) {
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
}

enum { F_DROP = 0, F_LIVE = 1, F_CULLED = 2 };

// a2 + cheap cone vs clear-direction map (p.cmap is never null: before any map
// is built it is the all-clear map, U = 1).  F_LIVE when the voxel may still
// change the AM, F_CULLED beyond reach, F_DROP otherwise.
__device__ __forceinline__ int fast_filter(const StreamParams& p, float4 q, uint32_t* sAM) {
    const float vx = q.x - p.px, vy = q.y - p.py, vz = q.z - p.pz, h = q.w;
    const float D2 = fmaf(vx, vx, fmaf(vy, vy, vz * vz));
    const float r2 = kSqrt3 * h;
    if (D2 <= 3.0001f * h * h) {
        // the pivot may lie in the closed box: then every orientation collides
        if (fabsf(vx) <= h && fabsf(vy) <= h && fabsf(vz) <= h) {
            fill_all(p, sAM);
            return F_DROP;
        }
        return F_LIVE;
    }
    const float invD = rsqrtf(D2);
    const float D = D2 * invD;
    if (D - r2 > p.cull_dist) return F_CULLED;
    const float Reff = reach_radius(p.tool, (D + r2) * (1.f + kRadRel));
    const float s = fmaf((Reff + r2) * invD, 1.f + 1.6e-5f, 1e-6f);
    // cube-map texel of v (cube_texel with an approximate reciprocal; the texel
    // radii carry 2e-5 rad of slack for the rounding at texel edges)
    const float ax = fabsf(vx), ay = fabsf(vy), az = fabsf(vz);
    const bool xm = ax >= fmaxf(ay, az);
    const bool ym = !xm && ay >= az;
    const float a = fmaxf(ax, fmaxf(ay, az));
    const float u = xm ? vy : vx;
    const float w = (xm || ym) ? vz : vy;
    const int face = xm ? (vx < 0.f) : (ym ? 2 + (vy < 0.f) : 4 + (vz < 0.f));
    const int T = p.cmapT;
    const float hs = 0.5f * (float)T;
    const float sc = hs * rcp_approx(a);
    const int iu = min(T - 1, max(0, __float2int_rz(fmaf(u, sc, hs))));
    const int iw = min(T - 1, max(0, __float2int_rz(fmaf(w, sc, hs))));
    const float U = __ldg(p.cmap + (face * T + iw) * T + iu);
    // U bounds cos(angle to the nearest clear cell) from above for every
    // direction of the texel: drop when cos(cheap cone) > U.
    const bool drop = (s < 1.f) ? (U < 0.f || U * U < 1.f - s * s) : (U < -1.5f);
    return drop ? F_DROP : F_LIVE;
}

// a3-a6 for one live voxel: both cones, rasterised row by row, band deferred.
__device__ __noinline__ void process_live(const StreamParams& p, unsigned int vidx, float4 q, uint32_t* sAM,
                                          const uint32_t* sRowFull, const float* sCos, const float* sSin,
                                          Counters cnt) {
    const ToolDev& T = p.tool;
    const GridDev& g = p.grid;
    const float vx = q.x - p.px, vy = q.y - p.py, vz = q.z - p.pz, h = q.w;
    const float D2 = vx * vx + vy * vy + vz * vz;
    const float D = sqrtf(D2);
    if (D <= kSqrt3 * h && fabsf(vx) <= h && fabsf(vy) <= h && fabsf(vz) <= h) return;  // filled already
    const float rxy = sqrtf(vx * vx + vy * vy);
    const float phv = atan2f(rxy, vz);
    // a4: the two cones (GETTOOLICA twice, Alg. 1)
    atomicAdd(cnt.c + CT_LIVE, 1u);
    const Cones c = tool_cones(D, h, T);
    if (c.cout > 1.f) return;
    const float ao = acosf(fmaxf(c.cout, -1.f));
    const int i0 = max(0, (int)ceilf((phv - ao - kRowSlack) * g.inv_dphi - 0.5f));
    const int i1 = min(g.m - 1, (int)floorf((phv + ao + kRowSlack) * g.inv_dphi - 0.5f));
    if (i0 > i1 || rows_all_full(sRowFull, i0, i1)) return;
    const float invD = 1.f / D;
    const float cphv = vz * invD, sphv = rxy * invD;
    const float gv = atan2f(vy, vx);
    const int W = g.W;
    unsigned int rows = 0;
    // a5: rasterise row by row (Alg. 1 L149-155 for all cells of a row at once)
    for (int i = i0; i <= i1; ++i) {
        if ((ld_vol_shared(sRowFull + (i >> 5)) >> (i & 31)) & 1u) continue;
        const float base = sCos[i] * cphv, den = sSin[i] * sphv;
        const Interval O = gamma_interval(c.cout, base, den, gv, +1, g);
        if (O.len == 0) continue;
        ++rows;
        const Interval In = gamma_interval(c.cin, base, den, gv, -1, g);
        const Interval X = gamma_interval(c.clo, base, den, gv, -1, g);
        for (int w = 0; w < W; ++w) {
            uint32_t ob = interval_bits(O, w, g.n);
            if (!ob) continue;
            const uint32_t xb = interval_bits(X, w, g.n);
            const uint32_t ib = interval_bits(In, w, g.n) & ~xb;
            ob &= ~xb;
            uint32_t* wp = sAM + i * W + w;
            uint32_t cur = ld_vol_shared(wp);
            if (ib & ~cur) {
                atomicOr(wp, ib);
                cur |= ib;
            }
            uint32_t band = ob & ~ib & ~cur;
            while (band) {
                const int b = __ffs(band) - 1;
                band &= band - 1u;
                push_band(p, sAM, vidx, q, i * g.n + (w << 5) + b, wp, 1u << b, cnt);
            }
        }
    }
    if (rows) atomicAdd(cnt.c + CT_ROWS, rows);
}

// a7 by one warp: OR the shared AM into the global AM (one atomicOr per word
// with bits the global AM may lack), OR the global AM back into shared memory,
// refresh the row-full bits.  Races between warps are benign: every update is
// an OR of bits that are certainly blocked.  Returns true when the AM is full.
__device__ __noinline__ bool warp_merge(const StreamParams& p, uint32_t* sAM, uint32_t* sShadow,
                                        uint32_t* sRowFull) {
    const int lane = threadIdx.x & 31;
    const int m = p.grid.m, W = p.grid.W, MW = m * W;
    for (int w = lane; w < MW; w += 32) {
        const uint32_t s = ld_vol_shared(sAM + w);
        const uint32_t sh = ld_vol_shared(sShadow + w);
        const uint32_t gv = (s & ~sh) ? (atomicOr(p.gam + w, s) | s) : ld_cg(p.gam + w);
        if (gv & ~s) atomicOr(sAM + w, gv);
        if (gv & ~sh) atomicOr(sShadow + w, gv | s);
    }
    __syncwarp();
    int nfull = 0;
    for (int i = lane; i < m; i += 32) {
        bool full = true;
        for (int w = 0; w < W; ++w)
            if (ld_vol_shared(sAM + i * W + w) != row_word_mask(w, p.grid.n)) full = false;
        if (full) {
            atomicOr(sRowFull + (i >> 5), 1u << (i & 31));
            ++nfull;
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) nfull += __shfl_xor_sync(0xffffffffu, nfull, o);
    return nfull == m;
}

// Dynamic shared memory of aica_stream_kernel for an m x n grid.
__host__ __device__ inline size_t stream_smem_bytes(int m, int W) {
    size_t b = (size_t)kWarps * kWStages * kChunk * sizeof(float4);  // per-warp TMA rings
    b += (size_t)kWarps * kWQ * sizeof(float4);                         // live queue voxels
    b += (size_t)kWarps * kWQ * sizeof(unsigned int);                   // live queue indices
    b += (size_t)(2 * m * W + ((m + 31) >> 5)) * sizeof(uint32_t);    // AM, shadow, row-full bits
    b += (size_t)2 * m * sizeof(float);                                 // cos / sin phi rows
    return b;
}

__global__ void __launch_bounds__(kThreads, 3) aica_stream_kernel(const __grid_constant__ StreamParams p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ uint64_t bar[kWarps][kWStages];
    __shared__ long long sChunk[kWarps][kWStages];
    __shared__ unsigned int sCnt[CT_COUNT];
    __shared__ unsigned long long sStreamed, sCulled, sPassed;
    __shared__ int sExit;
    // shared copy of the parameters for the out-of-line cold path (a reference
    // to the kernel parameter would make every call copy it to local memory)
    __shared__ StreamParams sP;
    if (threadIdx.x < (int)(sizeof(StreamParams) / 4))
        reinterpret_cast<unsigned int*>(&sP)[threadIdx.x] = reinterpret_cast<const unsigned int*>(&p)[threadIdx.x];
    const int m = p.grid.m;
    const int MW = m * p.grid.W;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    float4* ring = reinterpret_cast<float4*>(smem_raw) + warp * kWStages * kChunk;
    float4* sQv = reinterpret_cast<float4*>(smem_raw) + kWarps * kWStages * kChunk;
    unsigned int* sQi = reinterpret_cast<unsigned int*>(sQv + kWarps * kWQ);
    uint32_t* sAM = sQi + kWarps * kWQ;
    uint32_t* sShadow = sAM + MW;
    uint32_t* sRowFull = sShadow + MW;
    float* sCos = reinterpret_cast<float*>(sRowFull + ((m + 31) >> 5));
    float* sSin = sCos + m;
    float4* wQv = sQv + warp * kWQ;
    unsigned int* wQi = sQi + warp * kWQ;
    const Counters cnt{sCnt};

    for (int i = threadIdx.x; i < m; i += blockDim.x) {
        sCos[i] = p.tab[i];
        sSin[i] = p.tab[m + i];
    }
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        sAM[w] = 0u;
        sShadow[w] = 0u;
    }
    for (int w = threadIdx.x; w < ((m + 31) >> 5); w += blockDim.x) sRowFull[w] = 0u;
    if (threadIdx.x < CT_COUNT) sCnt[threadIdx.x] = 0u;
    if (threadIdx.x == 0) {
        sStreamed = sCulled = sPassed = 0ull;
        sExit = 0;
    }
    const long long nchunks = (p.N + kChunk - 1) / kChunk;
    long long nxt = 0, end = 0;  // lane 0's claimed chunk range
    auto claim = [&]() -> long long {
        if (nxt >= end) {
            nxt = (long long)atomicAdd(p.tile_ctr, (unsigned int)kSuper);
            end = nxt + kSuper;
        }
        return nxt++;
    };
    auto issue = [&](int s, long long c) {
        sChunk[warp][s] = c;
        if (c < nchunks) {
            const long long first = c * kChunk;
            const unsigned int bytes = (unsigned int)(min((long long)kChunk, p.N - first) * sizeof(float4));
            mbar_expect_tx(&bar[warp][s], bytes);
            tma_load_1d(ring + s * kChunk, p.vox + first, bytes, &bar[warp][s]);
        }
    };
    if (lane == 0) {
        for (int s = 0; s < kWStages; ++s) mbar_init(&bar[warp][s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int s = 0; s < kWStages; ++s) issue(s, claim());
    }
    __syncthreads();

    unsigned int phase = 0;      // bit s = parity of stage s
    unsigned int nculled = 0, npassed = 0;
    unsigned long long streamed = 0;
    int qn = 0;                  // live entries in this warp's queue (warp-uniform)
    int since = 0;
    int s = 0;
    bool early = false;
    for (;;) {
        const long long c = *reinterpret_cast<volatile long long*>(&sChunk[warp][s]);
        if (c >= nchunks) break;
        mbar_wait(&bar[warp][s], (phase >> s) & 1u);
        phase ^= 1u << s;
        const long long first = c * kChunk;
        const int cntv = (int)min((long long)kChunk, p.N - first);
        streamed += cntv;
        const float4* tv = ring + s * kChunk;
#pragma unroll
        for (int k = 0; k < kChunk / 32; ++k) {
            const int local = k * 32 + lane;
            int f = F_DROP;
            float4 q = make_float4(0.f, 0.f, 0.f, 0.f);
            if (local < cntv) {
                q = tv[local];
                f = fast_filter(p, q, sAM);
            }
            const unsigned int mlive = __ballot_sync(0xffffffffu, f == F_LIVE);
            nculled += __popc(__ballot_sync(0xffffffffu, f == F_CULLED));
            if (mlive) {
                npassed += __popc(mlive);
                if (f == F_LIVE) {
                    const int pos = qn + __popc(mlive & ((1u << lane) - 1u));
                    wQv[pos] = q;
                    wQi[pos] = (p.vbase + (unsigned int)(first + local)) | p.vtag;
                }
                qn += __popc(mlive);
                if (qn >= 32) {  // drain 32 entries, one per lane, then compact the rest
                    __syncwarp();
                    process_live(sP, wQi[lane], wQv[lane], sAM, sRowFull, sCos, sSin, cnt);
                    const int rest = qn - 32;
                    float4 rv;
                    unsigned int ri = 0;
                    if (lane < rest) {
                        rv = wQv[32 + lane];
                        ri = wQi[32 + lane];
                    }
                    __syncwarp();
                    if (lane < rest) {
                        wQv[lane] = rv;
                        wQi[lane] = ri;
                    }
                    __syncwarp();
                    qn = rest;
                }
            }
        }
        __syncwarp();  // the warp is done reading stage s
        if (lane == 0) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            issue(s, claim());
        }
        __syncwarp();
        if (++since >= p.refresh_tiles) {
            since = 0;
            if (warp_merge(sP, sAM, sShadow, sRowFull)) sExit = 1;
        }
        if (*reinterpret_cast<volatile int*>(&sExit)) {
            early = true;
            break;
        }
        s = (s + 1 == kWStages) ? 0 : s + 1;
    }
    if (lane < qn) process_live(sP, wQi[lane], wQv[lane], sAM, sRowFull, sCos, sSin, cnt);
    // an early exit may leave bulk copies in flight: wait for them before the
    // CTA retires (its shared memory must not be written after it exits)
    if (early) {
        for (int k = 0; k < kWStages; ++k)
            if (*reinterpret_cast<volatile long long*>(&sChunk[warp][k]) < nchunks)
                mbar_wait(&bar[warp][k], (phase >> k) & 1u);
    }
    if (lane == 0) {
        atomicAdd(&sCulled, (unsigned long long)nculled);
        atomicAdd(&sPassed, (unsigned long long)npassed);
        atomicAdd(&sStreamed, streamed);
    }
    // final flush of words that gained bits
    __syncthreads();
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        const uint32_t sv = sAM[w];
        if (sv & ~sShadow[w]) atomicOr(p.gam + w, sv);
    }
    if (threadIdx.x == 0) {
        atomicAdd(p.stats + ST_STREAMED, sStreamed);
        atomicAdd(p.stats + ST_CULLED, sCulled);
        atomicAdd(p.stats + ST_SKIPPED, sStreamed - sCulled - sPassed);
        atomicAdd(p.stats + ST_LIVE, (unsigned long long)sCnt[CT_LIVE]);
        atomicAdd(p.stats + ST_ROWS, (unsigned long long)sCnt[CT_ROWS]);
        atomicAdd(p.stats + ST_BAND, (unsigned long long)sCnt[CT_BAND]);
        atomicAdd(p.stats + ST_OVERFLOW, (unsigned long long)sCnt[CT_OVERFLOW]);
        if (early) atomicMax(p.stats + ST_EARLY, 1ULL);
    }
}

// Coarse levels: inner cones of the largest voxels, one warp per voxel with
// phi-rows across lanes, into a shared AM flushed to the global AM at the end.
// Voxels whose cheap cone holds no clear cell of p.cmap are skipped.
__global__ void __launch_bounds__(kThreads) coarse_kernel(const __grid_constant__ StreamParams p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    const GridDev& g = p.grid;
    const int m = g.m, W = g.W, MW = m * W;
    uint32_t* sAM = reinterpret_cast<uint32_t*>(smem_raw);
    float* sCos = reinterpret_cast<float*>(sAM + MW);
    float* sSin = sCos + m;
    for (int i = threadIdx.x; i < m; i += blockDim.x) {
        sCos[i] = p.tab[i];
        sSin[i] = p.tab[m + i];
    }
    for (int w = threadIdx.x; w < MW; w += blockDim.x) sAM[w] = 0u;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    const int B = p.tile;  // voxels per warp iteration: 1 (level 0, all live) or 32 (level 1, filtered)
    for (long long base = gw * B; base < p.N; base += nw * B) {
        const long long idx = base + lane;
        float4 q = make_float4(0.f, 0.f, 0.f, 1.f);
        int f = F_DROP;
        if (lane < B && idx < p.N) {
            q = p.vox[idx];
            f = fast_filter(p, q, sAM);
        }
        unsigned int live = __ballot_sync(0xffffffffu, f == F_LIVE);
        while (live) {
            const int src = __ffs(live) - 1;
            live &= live - 1u;
            const float4 v = make_float4(__shfl_sync(0xffffffffu, q.x, src), __shfl_sync(0xffffffffu, q.y, src),
                                         __shfl_sync(0xffffffffu, q.z, src), __shfl_sync(0xffffffffu, q.w, src));
            const float vx = v.x - p.px, vy = v.y - p.py, vz = v.z - p.pz, h = v.w;
            const float D = sqrtf(vx * vx + vy * vy + vz * vz);
            const float cin = inner_cone(D, h, p.tool);
            if (cin > 1.f) continue;
            const float rxy = sqrtf(vx * vx + vy * vy);
            const float phv = atan2f(rxy, vz);
            const float ai = acosf(fmaxf(cin, -1.f));
            const int i0 = max(0, (int)ceilf((phv - ai - kRowSlack) * g.inv_dphi - 0.5f));
            const int i1 = min(m - 1, (int)floorf((phv + ai + kRowSlack) * g.inv_dphi - 0.5f));
            const float invD = 1.f / D;
            const float cphv = vz * invD, sphv = rxy * invD;
            const float gv = atan2f(vy, vx);
            for (int i = i0 + lane; i <= i1; i += 32) {
                const Interval In = gamma_interval(cin, sCos[i] * cphv, sSin[i] * sphv, gv, -1, g);
                if (In.len == 0) continue;
                for (int w = 0; w < W; ++w) {
                    const uint32_t ib = interval_bits(In, w, g.n);
                    if (ib & ~ld_vol_shared(sAM + i * W + w)) atomicOr(sAM + i * W + w, ib);
                }
            }
        }
    }
    __syncthreads();
    for (int w = threadIdx.x; w < MW; w += blockDim.x) {
        const uint32_t sv = sAM[w];
        if (sv) atomicOr(p.gam + w, sv);
    }
}

}  // namespace am
