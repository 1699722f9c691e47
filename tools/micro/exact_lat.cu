// Microbenchmark + check: exact_hit (one thread) vs exact_hit_warp (one warp) -- latency in cycles
// and agreement on random (box, direction) cases around the paper's 3-cylinder tool.
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_icpp_chenktkv19_b200/csrc/geometry.cuh"
using namespace am;
__device__ unsigned int hash(unsigned int x) { x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x; }
__device__ float unif(unsigned int s) { return (hash(s) & 0xffffff) / 16777216.f; }
__global__ void lat(ToolDev T, float* io, long long* cyc, int warp) {
    float vx = io[0], vy = io[1], vz = io[2], h = io[3], dx = io[4], dy = io[5], dz = io[6];
    long long t0 = clock64();
    bool hit = false;
    for (int r = 0; r < 8; ++r) {
        hit |= warp ? exact_hit_warp(vx, vy, vz, h, dx, dy, dz, T) : exact_hit(vx, vy, vz, h, dx, dy, dz, T);
        vx += hit ? 1e-7f : 0.f;
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) { cyc[0] = (t1 - t0) / 8; io[8] = hit; }
}
__global__ void agree(ToolDev T, unsigned long long* bad, unsigned long long* hits, int n) {
    const int lane = threadIdx.x & 31;
    for (int i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n; i += (gridDim.x * blockDim.x) >> 5) {
        const unsigned s = 7919u * i;
        // directions near the box: a random box within 0..220 mm, a direction within ~0.6 rad of it
        const float D = 220.f * unif(s + 1), th = 3.14159f * unif(s + 2), ph = 6.2832f * unif(s + 3);
        const float vx = D * sinf(th) * cosf(ph), vy = D * sinf(th) * sinf(ph), vz = D * cosf(th);
        const float h = 0.01f + 3.f * unif(s + 4) * unif(s + 5);
        float dx = vx / (D + 1e-3f) + 0.6f * (unif(s + 6) - 0.5f), dy = vy / (D + 1e-3f) + 0.6f * (unif(s + 7) - 0.5f),
              dz = vz / (D + 1e-3f) + 0.6f * (unif(s + 8) - 0.5f);
        const float inv = rsqrtf(dx * dx + dy * dy + dz * dz);
        dx *= inv; dy *= inv; dz *= inv;
        const bool a = exact_hit(vx, vy, vz, h, dx, dy, dz, T);
        const bool b = exact_hit_warp(vx, vy, vz, h, dx, dy, dz, T);
        if (lane == 0) { if (a != b) atomicAdd(bad, 1ull); if (a) atomicAdd(hits, 1ull); }
    }
}
int main() {
    ToolDev T{};
    T.ncyl = 3;
    float R[3] = {6.35f, 6.225f, 20.f}, Hh[3] = {25.4f, 76.2f, 78.f};
    float z = 0;
    for (int c = 0; c < 3; ++c) { T.z0[c] = z; z += Hh[c]; T.z1[c] = z; T.R[c] = R[c]; }
    float hio[9] = {3.f, 2.f, 30.f, 0.01f, 0.f, 0.1f, 0.995f, 0, 0};
    float* io; long long* cyc; cudaMalloc(&io, 64); cudaMalloc(&cyc, 8);
    cudaMemcpy(io, hio, sizeof hio, cudaMemcpyHostToDevice);
    for (int w : {0, 1}) {
        lat<<<1, 32>>>(T, io, cyc, w);
        long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
        printf("%s: %lld cycles per test (%s)\n", w ? "exact_hit_warp" : "exact_hit (1 thread)", c, cudaGetErrorString(cudaGetLastError()));
    }
    unsigned long long *bad, *hits; cudaMalloc(&bad, 8); cudaMalloc(&hits, 8); cudaMemset(bad, 0, 8); cudaMemset(hits, 0, 8);
    const int n = 4 << 20;
    agree<<<1184, 256>>>(T, bad, hits, n);
    unsigned long long hb, hh; cudaMemcpy(&hb, bad, 8, cudaMemcpyDeviceToHost); cudaMemcpy(&hh, hits, 8, cudaMemcpyDeviceToHost);
    printf("agreement on %d random cases: %llu differ, %llu hits (%s)\n", n, hb, hh, cudaGetErrorString(cudaGetLastError()));
}
