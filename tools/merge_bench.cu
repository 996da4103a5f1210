// merge_bench.cu -- latency of one structured merge [R_a; R_b] -> R of the
// streaming skinny TSQR's tree (merge_group in tsqr_stream.cuh), one warp,
// clock64 per merge; and of the T-row write (stream_write_t).  Design study,
// not part of the library.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o tools/merge_bench tools/merge_bench.cu
#include <cstdio>
#include <cuda_runtime.h>
#include <type_traits>

#include "../paper_conf_ipps_andersonbdk11_b200/csrc/tsqr_stream.cuh"

using namespace caqr;

// Candidate: all 32 lanes busy.  lane = g * NC + k: column k, rows i = g + NG u
// (NG = 32 / NC row groups); every lane of column k keeps R_a's column k
// (redundantly), the row-j pivot entries travel by shuffles, the
// Householder scalars are computed redundantly by every lane (no shared
// memory, no __syncwarp inside the column loop).
// Round-1 merge: lane j computes the reflector, broadcasts it through shared
// memory; two __syncwarp per column.
template <typename T, int NC>
__device__ __forceinline__ void merge_smem(bool on, int k, const T* Ra, const T* Rb, int ld, int nb, T* Ro,
                                            T (&rb)[NC], T* G, int ldg, T* tau, T* bc) {
    T ra[NC];
#pragma unroll
    for (int i = 0; i < NC; ++i) {
        ra[i] = on ? Ra[i * ld + k] : T(0);
        rb[i] = (on && i < nb && i <= k) ? Rb[i * ld + k] : T(0);
    }
    __syncwarp();
#pragma unroll
    for (int j = 0; j < NC; ++j) {
        if (on && k == j) {
            T s0 = T(0), s1 = T(0);
#pragma unroll
            for (int i = 0; i <= j; i += 2) {
                s0 = fma(rb[i], rb[i], s0);
                if (i + 1 <= j) s1 = fma(rb[i + 1], rb[i + 1], s1);
            }
            T tj, beta, scale;
            householder_scalars(ra[j], s0 + s1, true, tj, beta, scale);
            ra[j] = beta;
#pragma unroll
            for (int i = 0; i <= j; ++i) {
                rb[i] *= scale;
                bc[i] = rb[i];
            }
            bc[NC] = tj;
            tau[j] = tj;
        }
        __syncwarp();
        if (on) {
            if (k > j) {
                const T tj = bc[NC];
                T s0 = ra[j], s1 = T(0);
#pragma unroll
                for (int i = 0; i <= j; i += 2) {
                    s0 = fma(bc[i], rb[i], s0);
                    if (i + 1 <= j) s1 = fma(bc[i + 1], rb[i + 1], s1);
                }
                const T f = tj * (s0 + s1);
                ra[j] -= f;
#pragma unroll
                for (int i = 0; i <= j; ++i) rb[i] = fma(-f, bc[i], rb[i]);
            } else if (k < j) {  // Gram entry (k, j): the R_a parts are unit vectors
                T gsum = T(0);
#pragma unroll
                for (int i = 0; i <= j; ++i) gsum = fma(rb[i], bc[i], gsum);
                G[k * ldg + j] = gsum;
            }
        }
        __syncwarp();
    }
    if (on)
#pragma unroll
        for (int i = 0; i < NC; ++i) Ro[i * ld + k] = i <= k ? ra[i] : T(0);
    __syncwarp();
}

// Candidate: the column loop NOT unrolled (small code: an instruction-cache
// cold merge fetches ~150 instructions instead of ~NC x 100); every row of
// the pivot column is shuffled (rows > j are zero), R_a's row j is kept in
// ra[0] by rotating the array each column.
template <typename T, int NC>
__device__ __forceinline__ void merge_rolled(bool on, int k, const T* Ra, const T* Rb, int ld, int nb, T* Ro,
                                             T (&rb)[NC], T* G, int ldg, T* tau) {
    T ra[NC];
#pragma unroll
    for (int i = 0; i < NC; ++i) {
        ra[i] = on ? Ra[i * ld + k] : T(0);
        rb[i] = (on && i < nb && i <= k) ? Rb[i * ld + k] : T(0);
    }
    __syncwarp();
#pragma unroll 1
    for (int j = 0; j < NC; ++j) {
        T y[NC];
#pragma unroll
        for (int i = 0; i < NC; ++i) y[i] = __shfl_sync(0xffffffffu, rb[i], j);
        const T al = __shfl_sync(0xffffffffu, ra[0], j);
        T s0 = T(0), s1 = T(0), d0 = T(0), d1 = T(0);
#pragma unroll
        for (int i = 0; i < NC; i += 2) {
            s0 = fma(y[i], y[i], s0);
            d0 = fma(y[i], rb[i], d0);
            s1 = fma(y[i + 1], y[i + 1], s1);
            d1 = fma(y[i + 1], rb[i + 1], d1);
        }
        const T d = d0 + d1;
        T tj, beta, scale;
        householder_scalars_nb(al, s0 + s1, tj, beta, scale);
        const bool diag = k == j;
        const T f = k > j ? tj * fma(scale, d, ra[0]) : T(0);
        const T r0 = diag ? beta : ra[0] - f;
        const T fs = f * scale;
#pragma unroll
        for (int i = 0; i < NC; ++i) rb[i] = diag ? rb[i] * scale : fma(-fs, y[i], rb[i]);
        if (on && k < j) G[k * ldg + j] = scale * d;
        if (on && diag) tau[j] = tj;
#pragma unroll
        for (int i = 0; i < NC - 1; ++i) ra[i] = ra[i + 1];
        ra[NC - 1] = r0;
    }
    if (on)
#pragma unroll
        for (int i = 0; i < NC; ++i) Ro[i * ld + k] = i <= k ? ra[i] : T(0);
    __syncwarp();
}

template <typename T, int NC>
__device__ __forceinline__ void merge_2d(const T* Ra, const T* Rb, int ld, int nb, T* Ro, T* V, T* G, int ldg,
                                         T* tau) {
    constexpr int NG = 32 / NC, RP = (NC + NG - 1) / NG;
    const int lane = threadIdx.x & 31, k = lane & (NC - 1), g = lane / NC;
    T ra[NC], rb[RP];
#pragma unroll
    for (int i = 0; i < NC; ++i) ra[i] = Ra[i * ld + k];
#pragma unroll
    for (int u = 0; u < RP; ++u) {
        const int i = g + NG * u;
        rb[u] = (i < NC && i < nb && i <= k) ? Rb[i * ld + k] : T(0);
    }
    __syncwarp();
#pragma unroll
    for (int j = 0; j < NC; ++j) {
        T y[RP], d = T(0);
#pragma unroll
        for (int u = 0; u < RP; ++u) {
            y[u] = __shfl_sync(0xffffffffu, rb[u], (lane & ~(NC - 1)) | j);
            d = fma(y[u], rb[u], d);
        }
#pragma unroll
        for (int o = NC; o < 32; o <<= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
        const T sg = __shfl_sync(0xffffffffu, d, j);
        const T al = __shfl_sync(0xffffffffu, ra[j], j);
        T tj, beta, scale;
        householder_scalars(al, sg, true, tj, beta, scale);
        if (k > j) {
            const T f = tj * fma(scale, d, ra[j]);
            ra[j] -= f;
            const T fs = f * scale;
#pragma unroll
            for (int u = 0; u < RP; ++u) rb[u] = fma(-fs, y[u], rb[u]);
        } else if (k == j) {
            ra[j] = beta;
#pragma unroll
            for (int u = 0; u < RP; ++u) rb[u] *= scale;
        } else if (g == 0) {
            G[k * ldg + j] = scale * d;
        }
        if (lane == 0) tau[j] = tj;
    }
    if (g == 0)
#pragma unroll
        for (int i = 0; i < NC; ++i) Ro[i * ld + k] = i <= k ? ra[i] : T(0);
#pragma unroll
    for (int u = 0; u < RP; ++u) {
        const int i = g + NG * u;
        if (i < NC) V[k * NC + i] = i <= k ? rb[u] : T(0);
    }
    __syncwarp();
}

template <int NC>
__global__ void bench(float* out, long long* cyc, int reps) {
    constexpr int LDR = NC + 1;
    __shared__ float Ra[NC * LDR], Rb[NC * LDR], G[NC * LDR], tau[NC], bc[2 * NC + 4], Tb[32 * 32];
    const int lane = threadIdx.x;
    for (int i = lane; i < NC * LDR; i += 32) {
        const int r = i / LDR, c = i % LDR;
        Ra[i] = c >= r ? 1.0f + 0.01f * (r * 7 + c * 3 % 5) : 0.0f;
        Rb[i] = c >= r ? 0.5f + 0.02f * (r * 3 + c * 5 % 7) : 0.0f;
    }
    __syncwarp();
    long long t0 = clock64();
    for (int it = 0; it < reps; ++it) {
        float rb[NC];
        merge_smem<float, NC>(lane < NC, lane, Ra, Rb, LDR, NC, Ra, rb, G, LDR, tau, bc);
        if (lane < NC) Rb[lane] = rb[0] * 0.5f + 0.5f;
        __syncwarp();
    }
    long long t1 = clock64();
    for (int it = 0; it < reps; ++it) {
        stream_write_t<float, NC>(lane < NC, lane, G, LDR, tau, NC, Tb);
        if (lane == 0) tau[0] += Tb[it & 31];
        __syncwarp();
    }
    long long t2 = clock64();
    __shared__ float V[NC * NC];
    for (int it = 0; it < reps; ++it) {
        merge_2d<float, NC>(Ra, Rb, LDR, NC, Ra, V, G, LDR, tau);
        if (lane < NC) Rb[lane] = V[lane * NC] * 0.5f + 0.5f;
        __syncwarp();
    }
    long long t3 = clock64();
    for (int it = 0; it < reps; ++it) {
        float rb[NC];
        merge_group<float, NC>(lane < NC, lane, Ra, Rb, LDR, NC, Ra, rb, G, LDR, tau);
        if (lane < NC) Rb[lane] = rb[0] * 0.5f + 0.5f;
        __syncwarp();
    }
    long long t4 = clock64();
    for (int it = 0; it < reps; ++it) {
        float rb[NC];
        merge_rolled<float, NC>(lane < NC, lane, Ra, Rb, LDR, NC, Ra, rb, G, LDR, tau);
        if (lane < NC) Rb[lane] = rb[0] * 0.5f + 0.5f;
        __syncwarp();
    }
    long long t5 = clock64();
    if (lane == 0) {
        cyc[4] = (t5 - t4) / reps;
        cyc[3] = (t4 - t3) / reps;
        cyc[0] = (t1 - t0) / reps;
        cyc[1] = (t2 - t1) / reps;
        cyc[2] = (t3 - t2) / reps;
    }
    out[lane] = Ra[lane % (NC * LDR)] + Tb[lane];
}

template <int NC>
__global__ void check(float* err) {
    constexpr int LDR = NC + 1;
    __shared__ float Ra[NC * LDR], Rb[NC * LDR], Ra2[NC * LDR], G[NC * LDR], G2[NC * LDR], tau[NC], tau2[NC],
        bc[2 * NC + 4], V[NC * NC], V1[NC * NC];
    const int lane = threadIdx.x;
    for (int i = lane; i < NC * LDR; i += 32) {
        const int r = i / LDR, c = i % LDR;
        Ra[i] = Ra2[i] = c >= r ? 1.0f + 0.37f * ((r * 7 + c * 3) % 5) - 0.9f * (c == r) : 0.0f;
        Rb[i] = c >= r ? -0.5f + 0.23f * ((r * 3 + c * 5) % 7) : 0.0f;
        G[i] = G2[i] = 0.0f;
    }
    __syncwarp();
    float rb[NC];
    merge_smem<float, NC>(lane < NC, lane, Ra, Rb, LDR, NC, Ra, rb, G, LDR, tau, bc);
    if (lane < NC)
        for (int i = 0; i < NC; ++i) V1[lane * NC + i] = i <= lane ? rb[i] : 0.0f;
    __syncwarp();
    merge_2d<float, NC>(Ra2, Rb, LDR, NC, Ra2, V, G2, LDR, tau2);
    __shared__ float Ra3[NC * LDR], G3[NC * LDR], tau3[NC], V3[NC * NC];
    for (int i = lane; i < NC * LDR; i += 32) {
        const int r = i / LDR, c = i % LDR;
        Ra3[i] = c >= r ? 1.0f + 0.37f * ((r * 7 + c * 3) % 5) - 0.9f * (c == r) : 0.0f;
        G3[i] = 0.0f;
    }
    __syncwarp();
    if (std::is_same<decltype(err), float*>::value && *reinterpret_cast<volatile int*>(&err[7]) == 1)
        merge_rolled<float, NC>(lane < NC, lane, Ra3, Rb, LDR, NC, Ra3, rb, G3, LDR, tau3);
    else
        merge_group<float, NC>(lane < NC, lane, Ra3, Rb, LDR, NC, Ra3, rb, G3, LDR, tau3);
    if (lane < NC)
        for (int i = 0; i < NC; ++i) V3[lane * NC + i] = i <= lane ? rb[i] : 0.0f;
    __syncwarp();
    if (lane == 0) {
        float e3 = 0;
        for (int i = 0; i < NC * LDR; ++i) {
            const int r = i / LDR, c = i % LDR;
            if (c < NC && c >= r) e3 = fmaxf(e3, fabsf(Ra[i] - Ra3[i]));
            if (c < NC && r < c) e3 = fmaxf(e3, fabsf(G[i] - G3[i]));
        }
        for (int i = 0; i < NC * NC; ++i) e3 = fmaxf(e3, fabsf(V3[i] - V1[i]));
        for (int i = 0; i < NC; ++i) e3 = fmaxf(e3, fabsf(tau[i] - tau3[i]));
        err[1] = e3;
        float e = 0;
        for (int i = 0; i < NC * LDR; ++i) {
            const int r = i / LDR, c = i % LDR;
            if (c < NC && c >= r) e = fmaxf(e, fabsf(Ra[i] - Ra2[i]));
            if (c < NC && r < c) e = fmaxf(e, fabsf(G[i] - G2[i]));
        }
        for (int i = 0; i < NC * NC; ++i) e = fmaxf(e, fabsf(V[i] - V1[i]));
        for (int i = 0; i < NC; ++i) e = fmaxf(e, fabsf(tau[i] - tau2[i]));
        *err = e;
    }
}

template <int NC>
void run() {
    {
        float* e;
        cudaMalloc(&e, 32);
        for (int mode = 0; mode < 2; ++mode) {
            cudaMemset(e, 0, 32);
            const int one = mode;
            cudaMemcpy(reinterpret_cast<char*>(e) + 28, &one, 4, cudaMemcpyHostToDevice);
            check<NC><<<1, 32>>>(e);
            float he[2] = {-1, -1};
            cudaMemcpy(he, e, 8, cudaMemcpyDeviceToHost);
            printf("NC=%2d: max |merge_2d - merge_smem| = %.3g, |%s - merge_smem| = %.3g\n", NC, he[0],
                   mode ? "merge_rolled" : "merge_group", he[1]);
        }
    }
    float* out;
    long long* cyc;
    cudaMalloc(&out, 128);
    cudaMalloc(&cyc, 64);
    bench<NC><<<1, 32>>>(out, cyc, 10);
    bench<NC><<<1, 32>>>(out, cyc, 1000);
    long long h[5];
    cudaMemcpy(h, cyc, 40, cudaMemcpyDeviceToHost);
    printf("NC=%2d: merge_smem %lld cycles, stream_write_t %lld cycles, merge_2d %lld, merge_group (shuffles) %lld, merge_rolled %lld cycles (%s)\n", NC, h[0], h[1], h[2], h[3], h[4],
           cudaGetErrorString(cudaGetLastError()));
}

int main() {
    run<4>();
    run<8>();
    run<16>();
    return 0;
}
