// umma_test.cu -- correctness probe of the tcgen05 wrappers in csrc/umma.cuh
// (descriptor layouts, K-major / MN-major operands, M = 64 / 128 TMEM layout,
// 3xTF32 accuracy).  Design study; not part of the library.
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_fp16.h>

#include "../paper_conf_ipps_andersonbdk11_b200/csrc/umma.cuh"

using namespace caqr;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

// byte offset of (x, k) in a K-major operand with LBO = 128, SBO = (K/4)*128
__host__ __device__ inline int kmaj(int x, int k, int K) { return (x % 8) * 16 + (k % 4) * 4 + (x / 8) * (K / 4) * 128 + (k / 4) * 128; }
// byte offset of (x, k) in an MN-major operand with SBO = 128, LBO = (X/4)*128
__host__ __device__ inline int mnmaj(int x, int k, int X) { return (x % 4) * 4 + (k % 8) * 16 + (x / 4) * 128 + (k / 8) * (X / 4) * 128; }

// D(M x N) = sum over nsplit products of A(M x K) B(K x N); A given as nA
// arrays (hi/lo), B as nB arrays; products listed in prod[] as (ia, ib).
template <int M, int N, int K>
__global__ void mma_kernel(const float* Ag, const float* Bg, int nA, int nB, int amn, const int* prod, int nprod,
                           float* Dout) {
    extern __shared__ __align__(128) unsigned char sm[];
    float* As = reinterpret_cast<float*>(sm);                 // nA * M*K
    float* Bs = As + nA * M * K;                              // nB * N*K
    __shared__ uint64_t mbar;
    __shared__ uint32_t tslot;
    const int tid = threadIdx.x;
    for (int a = 0; a < nA; ++a)
        for (int e = tid; e < M * K; e += blockDim.x) {
            const int m = e / K, k = e % K;
            const int off = amn ? mnmaj(m, k, M) : kmaj(m, k, K);
            *reinterpret_cast<float*>(reinterpret_cast<char*>(As + a * M * K) + off) = Ag[a * M * K + m * K + k];
        }
    for (int b = 0; b < nB; ++b)
        for (int e = tid; e < N * K; e += blockDim.x) {
            const int k = e / N, n = e % N;
            *reinterpret_cast<float*>(reinterpret_cast<char*>(Bs + b * N * K) + kmaj(n, k, K)) = Bg[b * K * N + k * N + n];
        }
    if (tid < 32) umma::tmem_alloc<128>(&tslot);
    if (tid == 0) umma::mbar_init(&mbar, 1);
    umma::fence_async_smem();
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    umma::fence_before_sync();
    __syncthreads();
    umma::fence_after_sync();
    const uint32_t tbase = tslot;
    if (tid == 0) {
        const uint32_t idesc = umma::idesc_tf32(M, N, amn != 0, false);
        bool acc = false;
        for (int pr = 0; pr < nprod; ++pr) {
            const float* Ab = As + prod[2 * pr] * M * K;
            const float* Bb = Bs + prod[2 * pr + 1] * N * K;
            for (int kk = 0; kk < K / 8; ++kk) {
                uint64_t ad, bd;
                if (amn == 1) ad = umma::sdesc(umma::smem_u32(Ab) + kk * (M / 4) * 128, (M / 4) * 128, 128);
                else if (amn == 2) ad = umma::sdesc(umma::smem_u32(Ab) + kk * (M / 4) * 128, 128, (M / 4) * 128);
                else ad = umma::sdesc(umma::smem_u32(Ab) + kk * 256, 128, (K / 4) * 128);
                bd = umma::sdesc(umma::smem_u32(Bb) + kk * 256, 128, (K / 4) * 128);
                umma::mma_tf32(tbase, ad, bd, idesc, acc);
                acc = true;
            }
        }
        umma::commit(&mbar);
    }
    umma::mbar_wait(&mbar, 0);
    umma::fence_after_sync();
    const int warp = tid >> 5, lane = tid & 31;
    for (int c0 = 0; c0 < N; c0 += 16) {
        float v[16];
        umma::tmem_ld16(tbase + ((uint32_t)(32 * warp) << 16) + c0, v);
        for (int i = 0; i < 16; ++i) Dout[(32 * warp + lane) * N + c0 + i] = v[i];
    }
    umma::fence_before_sync();
    __syncthreads();
    if (tid < 32) umma::tmem_free<128>(tbase);
}

static float tf32_rna(float x) {
    unsigned u; memcpy(&u, &x, 4);
    u = (u + 0x1000u) & 0xffffe000u;  // round half away (magnitude), fine for the test
    float r; memcpy(&r, &u, 4); return r;
}

template <int M, int N, int K>
void run(const char* name, int amn, bool split) {
    std::vector<float> A(M * K), B(K * N);
    unsigned s = 1234;
    auto rnd = [&]() { s = s * 1664525u + 1013904223u; return split ? ((s >> 8) & 0xffff) / 32768.f - 1.f : (float)((int)((s >> 16) % 7) - 3); };
    for (auto& x : A) x = rnd();
    for (auto& x : B) x = rnd();
    int nA = split ? 2 : 1, nB = split ? 2 : 1;
    std::vector<float> Ah(nA * M * K), Bh(nB * K * N);
    for (int i = 0; i < M * K; ++i) { float h = split ? tf32_rna(A[i]) : A[i]; Ah[i] = h; if (split) Ah[M * K + i] = A[i] - h; }
    for (int i = 0; i < K * N; ++i) { float h = split ? tf32_rna(B[i]) : B[i]; Bh[i] = h; if (split) Bh[K * N + i] = B[i] - h; }
    std::vector<int> prod = split ? std::vector<int>{1, 0, 0, 1, 0, 0} : std::vector<int>{0, 0};
    float *dA, *dB, *dD; int* dP;
    CK(cudaMalloc(&dA, Ah.size() * 4)); CK(cudaMalloc(&dB, Bh.size() * 4)); CK(cudaMalloc(&dD, 128 * N * 4)); CK(cudaMalloc(&dP, prod.size() * 4));
    CK(cudaMemcpy(dA, Ah.data(), Ah.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dB, Bh.data(), Bh.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dP, prod.data(), prod.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemset(dD, 0, 128 * N * 4));
    const size_t smem = (nA * M * K + nB * N * K) * 4;
    CK(cudaFuncSetAttribute(mma_kernel<M, N, K>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    mma_kernel<M, N, K><<<1, 128, smem>>>(dA, dB, nA, nB, amn, dP, (int)prod.size() / 2, dD);
    CK(cudaDeviceSynchronize());
    std::vector<float> D(128 * N);
    CK(cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost));
    // reference (double)
    std::vector<double> R(M * N, 0.0);
    for (int m = 0; m < M; ++m) for (int n = 0; n < N; ++n) { double a = 0; for (int k = 0; k < K; ++k) a += (double)A[m * K + k] * B[k * N + n]; R[m * N + n] = a; }
    // find, for each row m, the TMEM lane that holds it (first column match)
    int mapped = 0; double maxerr = 0, maxref = 0;
    std::vector<int> lane_of(M, -1);
    for (int m = 0; m < M; ++m) {
        for (int l = 0; l < 128; ++l) {
            bool ok = true;
            for (int n = 0; n < N && ok; ++n) ok = fabs(D[l * N + n] - R[m * N + n]) <= 1e-3 * (1 + fabs(R[m * N + n]));
            if (ok) { lane_of[m] = l; break; }
        }
        if (lane_of[m] >= 0) {
            ++mapped;
            for (int n = 0; n < N; ++n) { maxerr = fmax(maxerr, fabs(D[lane_of[m] * N + n] - R[m * N + n])); maxref = fmax(maxref, fabs(R[m * N + n])); }
        }
    }
    printf("%-34s M=%3d N=%3d K=%3d  rows mapped %d/%d  max|D-ref|/max|ref| = %.3e  lanes:", name, M, N, K, mapped, M, maxerr / (maxref + 1e-300));
    for (int m = 0; m < M; m += (M == 64 ? 4 : 16)) printf(" %d->%d", m, lane_of[m]);
    printf("\n");
    cudaFree(dA); cudaFree(dB); cudaFree(dD); cudaFree(dP);
}


// ---- kind::f16 probe: A (M x K) fp16, B (K x N) fp16; amn: 0 K-major, 1 MN-major (SBO=MN groups), 2 swapped
__host__ __device__ inline int kmaj16(int x, int k, int K) { return (x % 8) * 16 + (k % 8) * 2 + (x / 8) * (K / 8) * 128 + (k / 8) * 128; }
__host__ __device__ inline int mnmaj16(int x, int k, int X) { return (x % 8) * 2 + (k % 8) * 16 + (x / 8) * 128 + (k / 8) * (X / 8) * 128; }
template <int M, int N, int K>
__global__ void mma16_kernel(const float* Ag, const float* Bg, int amn, float* Dout) {
    extern __shared__ __align__(128) unsigned char sm[];
    __half* As = reinterpret_cast<__half*>(sm);
    __half* Bs = As + M * K;
    __shared__ uint64_t mbar;
    __shared__ uint32_t tslot;
    const int tid = threadIdx.x;
    for (int e = tid; e < M * K; e += blockDim.x) {
        const int m = e / K, k = e % K;
        const int off = amn ? mnmaj16(m, k, M) : kmaj16(m, k, K);
        *reinterpret_cast<__half*>(reinterpret_cast<char*>(As) + off) = __float2half(Ag[m * K + k]);
    }
    for (int e = tid; e < N * K; e += blockDim.x) {
        const int k = e / N, n = e % N;
        *reinterpret_cast<__half*>(reinterpret_cast<char*>(Bs) + kmaj16(n, k, K)) = __float2half(Bg[k * N + n]);
    }
    if (tid < 32) umma::tmem_alloc<128>(&tslot);
    if (tid == 0) umma::mbar_init(&mbar, 1);
    umma::fence_async_smem();
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    umma::fence_before_sync();
    __syncthreads();
    umma::fence_after_sync();
    const uint32_t tbase = tslot;
    if (tid == 0) {
        const uint32_t idesc = umma::idesc_f16(M, N, amn != 0, false);
        for (int kk = 0; kk < K / 16; ++kk) {
            uint64_t ad, bd;
            if (amn == 1) ad = umma::sdesc(umma::smem_u32(As) + kk * 2 * (M / 8) * 128, 2 * (M / 8) * 128 / 2, 128);
            else if (amn == 2) ad = umma::sdesc(umma::smem_u32(As) + kk * 2 * (M / 8) * 128, 128, (M / 8) * 128);
            else ad = umma::sdesc(umma::smem_u32(As) + kk * 256, 128, (K / 8) * 128);
            bd = umma::sdesc(umma::smem_u32(Bs) + kk * 256, 128, (K / 8) * 128);
            umma::mma_f16(tbase, ad, bd, idesc, kk > 0);
        }
        umma::commit(&mbar);
    }
    umma::mbar_wait(&mbar, 0);
    umma::fence_after_sync();
    const int warp = tid >> 5, lane = tid & 31;
    for (int c0 = 0; c0 < N; c0 += 16) {
        float v[16];
        umma::tmem_ld16(tbase + ((uint32_t)(32 * warp) << 16) + c0, v);
        for (int i = 0; i < 16; ++i) Dout[(32 * warp + lane) * N + c0 + i] = v[i];
    }
    umma::fence_before_sync();
    __syncthreads();
    if (tid < 32) umma::tmem_free<128>(tbase);
}

template <int M, int N, int K>
void run16(const char* name, int amn) {
    std::vector<float> A(M * K), B(K * N);
    unsigned s = 99;
    auto rnd = [&]() { s = s * 1664525u + 1013904223u; return (float)((int)((s >> 16) % 7) - 3); };
    for (auto& x : A) x = rnd();
    for (auto& x : B) x = rnd();
    float *dA, *dB, *dD;
    CK(cudaMalloc(&dA, A.size() * 4)); CK(cudaMalloc(&dB, B.size() * 4)); CK(cudaMalloc(&dD, 128 * N * 4));
    CK(cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemset(dD, 0, 128 * N * 4));
    const size_t smem = (M * K + N * K) * 2;
    CK(cudaFuncSetAttribute(mma16_kernel<M, N, K>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    mma16_kernel<M, N, K><<<1, 128, smem>>>(dA, dB, amn, dD);
    CK(cudaDeviceSynchronize());
    std::vector<float> D(128 * N);
    CK(cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost));
    int mapped = 0;
    std::vector<int> lane_of(M, -1);
    for (int m = 0; m < M; ++m) {
        for (int l = 0; l < 128; ++l) {
            bool ok = true;
            for (int n = 0; n < N && ok; ++n) { double r = 0; for (int k = 0; k < K; ++k) r += (double)A[m * K + k] * B[k * N + n]; ok = D[l * N + n] == r; }
            if (ok) { lane_of[m] = l; break; }
        }
        if (lane_of[m] >= 0) ++mapped;
    }
    printf("%-34s M=%3d N=%3d K=%3d  rows mapped exactly %d/%d  lanes:", name, M, N, K, mapped, M);
    for (int m = 0; m < M; m += 16) printf(" %d->%d", m, lane_of[m]);
    printf("\n");
    cudaFree(dA); cudaFree(dB); cudaFree(dD);
}

// ---- fp16x2 (hi/lo, power-of-two scaled) 3-term product, both GEMM shapes of the
// trailing update: W = V^T C (A = [Vh^T; Vl^T] K-major, M = 64) and
// dC = V W2 (A = V MN-major from the SAME buffer, M = 128).
__host__ __device__ inline int vbyte(int i, int r, int B) { return (i % 8) * 16 + (r % 8) * 2 + (i / 8) * (B / 8) * 128 + (r / 8) * 128; }
template <int B>  // rows
__global__ void fp16x2_kernel(const float* V, const float* C, const float* W2, float* Wout, float* dCout) {
    extern __shared__ __align__(128) unsigned char sm[];
    unsigned char* Vb = sm;                       // [hi: i 0..31 | lo: i 32..63] x B rows, fp16
    unsigned char* Cb = Vb + 64 * B * 2;          // C hi, C lo (16 cols x B rows each)
    unsigned char* Wb = Cb + 2 * 16 * B * 2;      // W2 hi, lo (16 cols x 32)
    __shared__ uint64_t mbar;
    __shared__ uint32_t tslot;
    __shared__ float cs[16], ws[16];
    const int tid = threadIdx.x;
    for (int e = tid; e < 32 * B; e += 128) {
        const int i = e / B, r = e % B;
        const float x = V[r * 32 + i] * 32768.f;
        const __half h = __float2half_rn(x), l = __float2half_rn(x - __half2float(h));
        *reinterpret_cast<__half*>(Vb + vbyte(i, r, B)) = h;
        *reinterpret_cast<__half*>(Vb + vbyte(i + 32, r, B)) = l;
    }
    if (tid < 16) {  // per-column power-of-two scales
        float m = 0.f; for (int r = 0; r < B; ++r) m = fmaxf(m, fabsf(C[r * 16 + tid]));
        int e = m > 0.f ? 14 - (int)(((__float_as_uint(m) >> 23) & 0xff) - 127) : 0;
        cs[tid] = __uint_as_float((uint32_t)(e + 127) << 23);
        float mw = 0.f; for (int i = 0; i < 32; ++i) mw = fmaxf(mw, fabsf(W2[i * 16 + tid]));
        int f = mw > 0.f ? 14 - (int)(((__float_as_uint(mw) >> 23) & 0xff) - 127) : 0;
        ws[tid] = __uint_as_float((uint32_t)(f + 127) << 23);
    }
    __syncthreads();
    for (int e = tid; e < 16 * B; e += 128) {
        const int n = e % 16, r = e / 16;
        const float x = C[r * 16 + n] * cs[n];
        const __half h = __float2half_rn(x), l = __float2half_rn(x - __half2float(h));
        const int off = (n % 8) * 16 + (r % 8) * 2 + (n / 8) * (B / 8) * 128 + (r / 8) * 128;
        *reinterpret_cast<__half*>(Cb + off) = h;
        *reinterpret_cast<__half*>(Cb + 16 * B * 2 + off) = l;
    }
    for (int e = tid; e < 16 * 32; e += 128) {
        const int n = e % 16, i = e / 16;
        const float x = W2[i * 16 + n] * ws[n];
        const __half h = __float2half_rn(x), l = __float2half_rn(x - __half2float(h));
        const int off = (n % 8) * 16 + (i % 8) * 2 + (n / 8) * 512 + (i / 8) * 128;
        *reinterpret_cast<__half*>(Wb + off) = h;
        *reinterpret_cast<__half*>(Wb + 1024 + off) = l;
    }
    if (tid < 32) umma::tmem_alloc<128>(&tslot);
    if (tid == 0) umma::mbar_init(&mbar, 1);
    umma::fence_async_smem();
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    umma::fence_before_sync();
    __syncthreads();
    umma::fence_after_sync();
    const uint32_t tb = tslot;
    const uint32_t SBOV = (B / 8) * 128;
    if (tid == 0) {
        // GEMM 1: D_W (M=64 x N=16) = [Vh^T; Vl^T] (Ch + Cl)
        const uint32_t id1 = umma::idesc_f16(64, 16, false, false);
        for (int kk = 0; kk < B / 16; ++kk)
            for (int h = 0; h < 2; ++h) {
                const uint64_t a = umma::sdesc(umma::smem_u32(Vb) + kk * 256, 128, SBOV);
                const uint64_t b = umma::sdesc(umma::smem_u32(Cb) + h * 16 * B * 2 + kk * 256, 128, (B / 8) * 128);
                umma::mma_f16(tb + 0, a, b, id1, kk > 0 || h > 0);
            }
        // GEMM 2: D_dC (M=128 x N=16) = Vh W2h + Vh W2l + Vl W2h (A = V MN-major: SBO = 128, LBO = SBOV)
        const uint32_t id2 = umma::idesc_f16(128, 16, true, false);
        const int pa[3] = {0, 0, 1}, pb[3] = {0, 1, 0};
        bool acc = false;
        for (int pr = 0; pr < 3; ++pr)
            for (int kk = 0; kk < 2; ++kk) {
                const uint64_t a = umma::sdesc(umma::smem_u32(Vb) + pa[pr] * 4 * SBOV + kk * 2 * SBOV, SBOV, 128);
                const uint64_t b = umma::sdesc(umma::smem_u32(Wb) + pb[pr] * 1024 + kk * 256, 128, 512);
                umma::mma_f16(tb + 32, a, b, id2, acc);
                acc = true;
            }
        umma::commit(&mbar);
    }
    umma::mbar_wait(&mbar, 0);
    umma::fence_after_sync();
    const int warp = tid >> 5, lane = tid & 31;
    {
        float v[16];
        umma::tmem_ld16(tb + ((uint32_t)(32 * warp) << 16) + 0, v);
        if (lane < 16) for (int n = 0; n < 16; ++n) Wout[(16 * warp + lane) * 16 + n] = v[n];
        umma::tmem_ld16(tb + ((uint32_t)(32 * warp) << 16) + 32, v);
        for (int n = 0; n < 16; ++n) dCout[(32 * warp + lane) * 16 + n] = v[n];
    }
    umma::fence_before_sync();
    __syncthreads();
    if (tid < 32) umma::tmem_free<128>(tb);
    if (tid < 16) { Wout[64 * 16 + tid] = cs[tid]; Wout[64 * 16 + 16 + tid] = ws[tid]; }
}

void run_fp16x2() {
    constexpr int B = 128;
    std::vector<float> V(B * 32), C(B * 16), W2(32 * 16);
    unsigned s = 7;
    auto rnd = [&]() { s = s * 1664525u + 1013904223u; return ((s >> 8) & 0xffff) / 32768.f - 1.f; };
    for (int r = 0; r < B; ++r) for (int i = 0; i < 32; ++i) V[r * 32 + i] = rnd() * (r == i ? 1.f : 0.3f);
    for (int r = 0; r < B; ++r) for (int n = 0; n < 16; ++n) C[r * 16 + n] = rnd() * (n < 8 ? 1000.f : 0.001f);
    for (auto& x : W2) x = rnd() * 37.f;
    float *dV, *dC, *dW, *dWo, *ddC;
    CK(cudaMalloc(&dV, V.size() * 4)); CK(cudaMalloc(&dC, C.size() * 4)); CK(cudaMalloc(&dW, W2.size() * 4));
    CK(cudaMalloc(&dWo, (64 * 16 + 32) * 4)); CK(cudaMalloc(&ddC, 128 * 16 * 4));
    CK(cudaMemcpy(dV, V.data(), V.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dC, C.data(), C.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dW, W2.data(), W2.size() * 4, cudaMemcpyHostToDevice));
    const size_t smem = 64 * B * 2 + 2 * 16 * B * 2 + 2048;
    CK(cudaFuncSetAttribute(fp16x2_kernel<B>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    fp16x2_kernel<B><<<1, 128, smem>>>(dV, dC, dW, dWo, ddC);
    CK(cudaDeviceSynchronize());
    std::vector<float> Wo(64 * 16 + 32), dCo(128 * 16);
    CK(cudaMemcpy(Wo.data(), dWo, Wo.size() * 4, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(dCo.data(), ddC, dCo.size() * 4, cudaMemcpyDeviceToHost));
    double ew = 0, nw = 0, ec = 0, nc = 0;
    for (int n = 0; n < 16; ++n) {
        double colmax = 0, err = 0;
        for (int i = 0; i < 32; ++i) {
            double ref = 0; for (int r = 0; r < B; ++r) ref += (double)V[r * 32 + i] * C[r * 16 + n];
            // M=64 layout: row i (hi part) in lane 16*(i/16)... stored by warp (i/16) lane (i%16): Wout row 16*w + l
            const double got = ((double)Wo[i * 16 + n] + (double)Wo[(i + 32) * 16 + n]) / (32768.0 * Wo[64 * 16 + n]);
            err = fmax(err, fabs(got - ref)); colmax = fmax(colmax, fabs(ref));
        }
        ew = fmax(ew, err / (colmax + 1e-300));
        double cmax = 0, cerr = 0;
        for (int r = 0; r < B; ++r) {
            double ref = 0; for (int i = 0; i < 32; ++i) ref += (double)V[r * 32 + i] * W2[i * 16 + n];
            const double got = (double)dCo[r * 16 + n] / (32768.0 * Wo[64 * 16 + 16 + n]);
            cerr = fmax(cerr, fabs(got - ref)); cmax = fmax(cmax, fabs(ref));
        }
        ec = fmax(ec, cerr / (cmax + 1e-300));
    }
    printf("fp16x2 3-term: W = V^T C (M=64 K-major) max colwise rel err %.3e;  dC = V W2 (M=128 MN-major, same V buffer) %.3e\n", ew, ec);
}

int main() {
    setvbuf(stdout, NULL, _IONBF, 0);
    run<128, 32, 32>("K-major A, integer", 0, false);
    run<64, 32, 32>("K-major A, integer", 0, false);
    run<128, 32, 32>("MN-major A, integer", 1, false);
    run<64, 32, 32>("MN-major A, integer", 1, false);
    run<128, 16, 64>("K-major A, integer, N=16", 0, false);
    run<128, 32, 32>("MN-major A (LBO/SBO swapped)", 2, false);
    run<64, 32, 32>("MN-major A (LBO/SBO swapped)", 2, false);
    run16<128, 32, 64>("f16 K-major A", 0);
    run16<128, 32, 64>("f16 MN-major A", 1);
    run16<64, 16, 64>("f16 MN-major A", 1);
    run_fp16x2();
    run<128, 32, 128>("3xTF32 K-major", 0, true);
    run<64, 32, 192>("3xTF32 K-major", 0, true);
    run<128, 32, 32>("3xTF32 MN-major (swapped)", 2, true);
    return 0;
}
