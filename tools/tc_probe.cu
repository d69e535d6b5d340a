// tc_probe.cu -- standalone probe of tcgen05 conventions used by tc.cu:
// A operand in TMEM (tcgen05.st 32x32b), B in shared memory (K-major
// SWIZZLE_NONE canonical layout), kind::tf32, M = 128, N = 32, K = 8 x KB.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -o tc_probe tools/tc_probe.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cmath>
#include <vector>

#define N 32
#define KB 4
#define KK (8 * KB)

__device__ __forceinline__ uint64_t desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
    d |= 1ull << 46;
    return d;
}

__global__ void probe(const float* A /*128 x KK*/, const float* B /*KK x N (row kk)*/, float* D /*128 x N*/, int mode) {
    __shared__ __align__(1024) float sB[N * KK];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tslot;
    const int tid = threadIdx.x, warp = tid >> 5;
    // B^T (N rows x KK) in K-major canonical: (n>>3)*SBO + (kk>>2)*128 + (n&7)*16 + (kk&3)*4
    const uint32_t SBO = (KK / 4) * 128;
    for (int e = tid; e < N * KK; e += blockDim.x) {
        int n = e / KK, kk = e % KK;
        uint32_t off = (n >> 3) * SBO + (kk >> 2) * 128 + (n & 7) * 16 + (kk & 3) * 4;
        sB[off / 4] = B[kk * N + n];
    }
    uint32_t sbar = (uint32_t)__cvta_generic_to_shared(&bar);
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sbar));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(
            (uint32_t)__cvta_generic_to_shared(&tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tb = tslot;
    // A row tid -> TMEM lane tid, columns [64, 64+KK)
    const uint32_t ta = tb + ((uint32_t)(warp * 32) << 16) + 64;
    for (int c0 = 0; c0 < KK; c0 += 8) {
        uint32_t v[8];
        for (int j = 0; j < 8; ++j) v[j] = __float_as_uint(A[tid * KK + c0 + j]);
        asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(ta + c0),
                     "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]));
    }
    asm volatile("tcgen05.wait::st.sync.aligned;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    if (tid == 0) {
        const uint32_t sb = (uint32_t)__cvta_generic_to_shared(sB);
        for (int kb = 0; kb < KB; ++kb) {
            uint64_t bd = desc(sb + kb * 256, 128, SBO);
            uint32_t acc = kb > 0;
            uint32_t a_t = tb + 64 + (uint32_t)(kb * 8 * mode);  // mode: column step per k-block (probe)
            asm volatile(
                "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tb),
                "r"(a_t), "l"(bd), "r"(idesc), "r"(acc));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(sbar));
    }
    asm volatile(
        "{\n\t.reg .pred d;\n\tW: mbarrier.try_wait.parity.shared::cta.b64 d, [%0], 0;\n\t@!d bra W;\n\t}" ::"r"(sbar));
    asm volatile("tcgen05.fence::after_thread_sync;");
    uint32_t v[32];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(tb + ((uint32_t)(warp * 32) << 16)));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    for (int j = 0; j < 32; ++j) D[tid * N + j] = __uint_as_float(v[j]);
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tb));
}

int main() {
    std::vector<float> A(128 * KK), B(KK * N), D(128 * N), R(128 * N, 0.f);
    srand(1);
    // tf32-exact small integers so the product is exact
    for (auto& x : A) x = (float)(rand() % 7 - 3);
    for (auto& x : B) x = (float)(rand() % 5 - 2);
    for (int m = 0; m < 128; ++m)
        for (int n = 0; n < N; ++n)
            for (int k = 0; k < KK; ++k) R[m * N + n] += A[m * KK + k] * B[k * N + n];
    float *dA, *dB, *dD;
    cudaMalloc(&dA, A.size() * 4);
    cudaMalloc(&dB, B.size() * 4);
    cudaMalloc(&dD, D.size() * 4);
    cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice);
    for (int mode = 0; mode <= 1; ++mode) {
        cudaMemset(dD, 0, D.size() * 4);
        probe<<<1, 128>>>(dA, dB, dD, mode);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) {
            printf("mode %d: CUDA error %s\n", mode, cudaGetErrorString(e));
            return 1;
        }
        cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
        double err = 0;
        for (size_t i = 0; i < D.size(); ++i) err = fmax(err, fabs(D[i] - R[i]));
        printf("TS probe mode %d (A column step %d per k-block): max err %g  D[0]=%g R[0]=%g\n", mode, 8 * mode, err,
               D[0], R[0]);
    }
    return 0;
}
