// pf_bench.cu -- microbenchmark of structured panel-factorization layouts
// (design study for the round-2 kernels; not part of the library).
//
// One "panel step" = the structured Householder QR of [Rhead; X] where X is a
// ROWS x NC tile and Rhead the NC x NC upper triangle of the chain's running R
// (reflector j = [e_j on R row j; v_j on the tile rows]).
//
// Mode A (cq): thread t owns column c = t / NQ and row segment q = t % NQ
//   (SEG = ROWS / NQ rows in registers); the pivot v_j is broadcast through
//   shared memory, dots are reduced over the NQ owner threads by shuffles;
//   one CTA barrier per column.
// Mode B (warp): one warp owns the whole tile (lane = rows l + 32 i, all NC
//   columns in registers); per column one multi-value warp reduction through
//   shared memory; no CTA barrier.
//
// Reports cycles per panel step per CTA for k CTAs per SM (throughput) .
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

__device__ __forceinline__ void rsq(float s, float& r, float& sq) {
    float y = rsqrtf(s);
    const float h = 0.5f * s * y;
    y = fmaf(-h, y, 1.5f) * y;
    r = y;
    const float q = s * y;
    sq = fmaf(fmaf(-q, q, s), 0.5f * y, q);
}
__device__ __forceinline__ float rcpr(float d) {
    float y = __fdividef(1.0f, d);
    return fmaf(fmaf(-d, y, 1.0f), y, y);
}

template <int NC, int NQ, int SEG>
__global__ void __launch_bounds__(NC* NQ) cq_kernel(const float* __restrict__ X0, float* out, int iters,
                                                      long long* cyc) {
    constexpr int ROWS = NQ * SEG;
    constexpr int SP = SEG + 4;  // padded segment stride in vbuf
    __shared__ __align__(16) float vbuf[2][NQ * SP];
    __shared__ float head[NC][NC + 1];
    __shared__ float stau[2];
    const int t = threadIdx.x, c = t / NQ, q = t % NQ;
    const unsigned gm = ((NQ >= 32) ? 0xffffffffu : ((1u << NQ) - 1u)) << ((t & 31) & ~(NQ - 1));
    const float* src = X0 + (size_t)blockIdx.x * ROWS * NC;
    float x[SEG];
    long long t0 = clock64();
    float acc = 0.f;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < SEG; ++i) x[i] = __ldg(src + (size_t)c * ROWS + q * SEG + i);
        for (int e = t; e < NC * NC; e += NC * NQ) head[e / NC][e % NC] = (e / NC == e % NC) ? 1.5f : 0.25f;
        __syncthreads();
        // pivot 0
        if (c == 0) {
            float s0 = 0, s1 = 0, s2 = 0, s3 = 0;
#pragma unroll
            for (int i = 0; i < SEG; i += 4) {
                s0 = fmaf(x[i], x[i], s0); s1 = fmaf(x[i + 1], x[i + 1], s1);
                s2 = fmaf(x[i + 2], x[i + 2], s2); s3 = fmaf(x[i + 3], x[i + 3], s3);
            }
            float sg = (s0 + s1) + (s2 + s3);
#pragma unroll
            for (int o = 1; o < NQ; o <<= 1) sg += __shfl_xor_sync(gm, sg, o);
            const float al = head[0][0];
            float rmu, mu;
            rsq(fmaf(al, al, sg), rmu, mu);
            const float tau = fmaf(fabsf(al), rmu, 1.f);
            const float sc = copysignf(rcpr(fabsf(al) + mu), al);
#pragma unroll
            for (int i = 0; i < SEG; ++i) x[i] *= sc;
#pragma unroll
            for (int i = 0; i < SEG; i += 4)
                *reinterpret_cast<float4*>(&vbuf[0][q * SP + i]) = make_float4(x[i], x[i + 1], x[i + 2], x[i + 3]);
            if (q == 0) { stau[0] = tau; head[0][0] = -copysignf(mu, al); }
        }
        __syncthreads();
        for (int j = 0; j < NC; ++j) {
            const int b = j & 1;
            if (c > j) {
                const float tau = stau[b];
                float v[SEG];
#pragma unroll
                for (int i = 0; i < SEG; i += 4) {
                    const float4 f = *reinterpret_cast<const float4*>(&vbuf[b][q * SP + i]);
                    v[i] = f.x; v[i + 1] = f.y; v[i + 2] = f.z; v[i + 3] = f.w;
                }
                float d0 = 0, d1 = 0, d2 = 0, d3 = 0;
#pragma unroll
                for (int i = 0; i < SEG; i += 4) {
                    d0 = fmaf(v[i], x[i], d0); d1 = fmaf(v[i + 1], x[i + 1], d1);
                    d2 = fmaf(v[i + 2], x[i + 2], d2); d3 = fmaf(v[i + 3], x[i + 3], d3);
                }
                float d = (d0 + d1) + (d2 + d3);
#pragma unroll
                for (int o = 1; o < NQ; o <<= 1) d += __shfl_xor_sync(gm, d, o);
                const float hs = head[j][c];
                const float st = tau * (hs + d);
                if (q == 0) head[j][c] = hs - st;
#pragma unroll
                for (int i = 0; i < SEG; ++i) x[i] = fmaf(-st, v[i], x[i]);
                if (c == j + 1) {
                    float s0 = 0, s1 = 0, s2 = 0, s3 = 0;
#pragma unroll
                    for (int i = 0; i < SEG; i += 4) {
                        s0 = fmaf(x[i], x[i], s0); s1 = fmaf(x[i + 1], x[i + 1], s1);
                        s2 = fmaf(x[i + 2], x[i + 2], s2); s3 = fmaf(x[i + 3], x[i + 3], s3);
                    }
                    float sg = (s0 + s1) + (s2 + s3);
#pragma unroll
                    for (int o = 1; o < NQ; o <<= 1) sg += __shfl_xor_sync(gm, sg, o);
                    const float al = head[j + 1][j + 1];
                    float rmu, mu;
                    rsq(fmaf(al, al, sg), rmu, mu);
                    const float tau2 = fmaf(fabsf(al), rmu, 1.f);
                    const float sc = copysignf(rcpr(fabsf(al) + mu), al);
#pragma unroll
                    for (int i = 0; i < SEG; ++i) x[i] *= sc;
#pragma unroll
                    for (int i = 0; i < SEG; i += 4)
                        *reinterpret_cast<float4*>(&vbuf[b ^ 1][q * SP + i]) =
                            make_float4(x[i], x[i + 1], x[i + 2], x[i + 3]);
                    if (q == 0) { stau[b ^ 1] = tau2; head[j + 1][j + 1] = -copysignf(mu, al); }
                }
            }
            __syncthreads();
        }
#pragma unroll
        for (int i = 0; i < SEG; ++i) acc += x[i];
    }
    long long t1 = clock64();
    if (t == 0) cyc[blockIdx.x] = t1 - t0;
    out[blockIdx.x * blockDim.x + t] = acc + head[c % NC][c % NC];
}

template <int NC, int RL, int J>
__device__ __forceinline__ void wstep(float (&x)[RL][NC], float* scr, float* tot, float (*head)[NC + 1], int lane) {
    if constexpr (J < NC) {
        constexpr int j = J;

            // partial products of column j with columns j..NC-1 over this lane's rows
#pragma unroll
            for (int c = j; c < NC; ++c) {
                float a = 0.f;
#pragma unroll
                for (int i = 0; i < RL; ++i) a = fmaf(x[i][j], x[i][c], a);
                scr[lane * (NC + 4) + c] = a;
            }
            __syncwarp();
            if (lane >= j && lane < NC) {
                float a0 = 0, a1 = 0, a2 = 0, a3 = 0;
#pragma unroll
                for (int r = 0; r < 32; r += 4) {
                    a0 += scr[(r + 0) * (NC + 4) + lane]; a1 += scr[(r + 1) * (NC + 4) + lane];
                    a2 += scr[(r + 2) * (NC + 4) + lane]; a3 += scr[(r + 3) * (NC + 4) + lane];
                }
                tot[lane] = (a0 + a1) + (a2 + a3);
            }
            __syncwarp();
            const float sg = tot[j];
            const float al = head[j][j];
            float rmu, mu;
            rsq(fmaf(al, al, sg), rmu, mu);
            const float tau = fmaf(fabsf(al), rmu, 1.f);
            const float sc = copysignf(rcpr(fabsf(al) + mu), al);
#pragma unroll
            for (int i = 0; i < RL; ++i) x[i][j] *= sc;
#pragma unroll
            for (int c = j + 1; c < NC; ++c) {
                const float hs = head[j][c];
                const float st = tau * fmaf(sc, tot[c], hs);
#pragma unroll
                for (int i = 0; i < RL; ++i) x[i][c] = fmaf(-st, x[i][j], x[i][c]);
                if (lane == 0) head[j][c] = hs - st;
            }
            if (lane == 0) head[j][j] = -copysignf(mu, al);
            __syncwarp();
                wstep<NC, RL, J + 1>(x, scr, tot, head, lane);
    }
}

// Mode B: one warp per tile, RL rows per lane (ROWS = 32 RL), NC <= 32 columns.
template <int NC, int RL>
__global__ void __launch_bounds__(32) warp_kernel(const float* __restrict__ X0, float* out, int iters,
                                                  long long* cyc) {
    constexpr int ROWS = 32 * RL;
    __shared__ __align__(16) float scr[32 * (NC + 4)];
    __shared__ __align__(16) float tot[NC];
    __shared__ float head[NC][NC + 1];
    const int lane = threadIdx.x;
    const float* src = X0 + (size_t)blockIdx.x * ROWS * NC;
    float x[RL][NC];
    long long t0 = clock64();
    float acc = 0.f;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int c = 0; c < NC; ++c)
#pragma unroll
            for (int i = 0; i < RL; ++i) x[i][c] = __ldg(src + (size_t)c * ROWS + lane + 32 * i);
        for (int e = lane; e < NC * NC; e += 32) head[e / NC][e % NC] = (e / NC == e % NC) ? 1.5f : 0.25f;
        __syncwarp();
wstep<NC, RL, 0>(x, scr, tot, head, lane);
#pragma unroll
        for (int c = 0; c < NC; ++c)
#pragma unroll
            for (int i = 0; i < RL; ++i) acc += x[i][c];
    }
    long long t1 = clock64();
    if (lane == 0) cyc[blockIdx.x] = t1 - t0;
    out[blockIdx.x * 32 + lane] = acc;
}

template <typename K>
void run(const char* name, K kern, int threads, int rows, int nc, int per_sm, int iters) {
    const int nsm = 148, grid = nsm * per_sm;
    float *X, *out;
    long long* cyc;
    CK(cudaMalloc(&X, (size_t)grid * rows * nc * 4));
    CK(cudaMalloc(&out, (size_t)grid * 1024 * 4));
    CK(cudaMalloc(&cyc, grid * 8));
    // deterministic pseudo-random fill
    float* h = (float*)malloc((size_t)grid * rows * nc * 4);
    unsigned s = 12345;
    for (size_t i = 0; i < (size_t)grid * rows * nc; ++i) { s = s * 1664525u + 1013904223u; h[i] = ((s >> 8) & 0xffff) / 65536.f - 0.5f; }
    CK(cudaMemcpy(X, h, (size_t)grid * rows * nc * 4, cudaMemcpyHostToDevice));
    kern<<<grid, threads>>>(X, out, 2, cyc);
    CK(cudaDeviceSynchronize());
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<<<grid, threads>>>(X, out, iters, cyc);
    cudaEventRecord(e1);
    CK(cudaDeviceSynchronize());
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    long long* hc = (long long*)malloc(grid * 8);
    CK(cudaMemcpy(hc, cyc, grid * 8, cudaMemcpyDeviceToHost));
    double mean = 0; for (int i = 0; i < grid; ++i) mean += hc[i]; mean /= grid;
    // rows*columns processed per SM per cycle
    const double steps_per_sm = (double)per_sm * iters;
    fflush(stdout); printf("%-28s rows=%3d nc=%2d ctas/SM=%2d  cyc/panel/CTA=%8.0f  cyc/col=%6.0f  SM-throughput: %.1f cyc per panel  (%.3f ms)\n",
           name, rows, nc, per_sm, mean / iters, mean / iters / nc, ms * 1.9e6 / steps_per_sm, ms);
    cudaFree(X); cudaFree(out); cudaFree(cyc); free(h); free(hc);
}

int main() {
    setvbuf(stdout, NULL, _IONBF, 0);
    const int it = 200;
    for (int k : {1, 2, 4, 8}) run("cq NC32 NQ4 SEG32", cq_kernel<32, 4, 32>, 128, 128, 32, k, it);
    for (int k : {1, 2, 4, 8}) run("cq NC32 NQ8 SEG16", cq_kernel<32, 8, 16>, 256, 128, 32, k, it);
    for (int k : {1, 2, 4}) run("cq NC64 NQ4 SEG32", cq_kernel<64, 4, 32>, 256, 128, 64, k, it);
    for (int k : {1, 2, 4}) run("cq NC32 NQ4 SEG64", cq_kernel<32, 4, 64>, 128, 256, 32, k, it);
    for (int k : {1, 2, 4}) run("cq NC32 NQ8 SEG32", cq_kernel<32, 8, 32>, 256, 256, 32, k, it);
    for (int k : {1, 2, 4}) run("cq NC64 NQ2 SEG32", cq_kernel<64, 2, 32>, 128, 64, 64, k, it);
    for (int k : {1, 4, 8, 16}) run("warp NC32 RL4", warp_kernel<32, 4>, 32, 128, 32, k, it);
    for (int k : {1, 4, 8, 16}) run("warp NC32 RL2", warp_kernel<32, 2>, 32, 64, 32, k, it);
    for (int k : {1, 4, 8, 16}) run("warp NC16 RL4", warp_kernel<16, 4>, 32, 128, 16, k, it);
    return 0;
}
