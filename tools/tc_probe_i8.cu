// tc_probe_i8.cu -- standalone probe of tcgen05.mma.kind::i8 (SS, K-major
// SWIZZLE_NONE canonical layout, M = 128, N = 32, K = 32 per instruction).
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>

#define N 32
#define KK 64

__device__ __forceinline__ uint64_t desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}

__global__ void probe(const int8_t* A, const int8_t* B, int* D, int a_signed, int b_signed) {
    __shared__ __align__(1024) int8_t sA[128 * KK];
    __shared__ __align__(1024) int8_t sB[N * KK];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tslot;
    const int tid = threadIdx.x, warp = tid >> 5;
    const uint32_t SBO = (KK / 16) * 128;
    for (int e = tid; e < 128 * KK; e += blockDim.x) {
        int r = e / KK, k = e % KK;
        sA[(r >> 3) * SBO + (k >> 4) * 128 + (r & 7) * 16 + (k & 15)] = A[r * KK + k];
    }
    for (int e = tid; e < N * KK; e += blockDim.x) {
        int n = e / KK, k = e % KK;
        sB[(n >> 3) * SBO + (k >> 4) * 128 + (n & 7) * 16 + (k & 15)] = B[k * N + n];
    }
    uint32_t sbar = (uint32_t)__cvta_generic_to_shared(&bar);
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sbar));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(
            (uint32_t)__cvta_generic_to_shared(&tslot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tb = tslot;
    const uint32_t idesc = (2u << 4) | ((uint32_t)a_signed << 7) | ((uint32_t)b_signed << 10) |
                           ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    if (tid == 0) {
        const uint32_t sa = (uint32_t)__cvta_generic_to_shared(sA), sb = (uint32_t)__cvta_generic_to_shared(sB);
        for (int ks = 0; ks < KK / 32; ++ks) {
            uint64_t ad = desc(sa + ks * 256, 128, SBO), bd = desc(sb + ks * 256, 128, SBO);
            uint32_t acc = ks > 0;
            asm volatile(
                "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(tb),
                "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
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
    for (int j = 0; j < 32; ++j) D[tid * N + j] = (int)v[j];
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(tb));
}

int main() {
    std::vector<int8_t> A(128 * KK), B(KK * N);
    std::vector<int> D(128 * N);
    srand(3);
    int8_t *dA, *dB;
    int* dD;
    cudaMalloc(&dA, A.size());
    cudaMalloc(&dB, B.size());
    cudaMalloc(&dD, D.size() * 4);
    for (int as = 0; as <= 1; ++as)
        for (int bs = 0; bs <= 1; ++bs) {
            for (auto& x : A) x = (int8_t)(as ? (rand() % 256 - 128) : (rand() % 256));
            for (auto& x : B) x = (int8_t)(bs ? (rand() % 256 - 128) : (rand() % 256));
            cudaMemcpy(dA, A.data(), A.size(), cudaMemcpyHostToDevice);
            cudaMemcpy(dB, B.data(), B.size(), cudaMemcpyHostToDevice);
            cudaMemset(dD, 0, D.size() * 4);
            probe<<<1, 128>>>(dA, dB, dD, as, bs);
            cudaError_t e = cudaDeviceSynchronize();
            if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
            cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
            long long maxerr = 0;
            long long r00 = 0;
            for (int m = 0; m < 128; ++m)
                for (int n = 0; n < N; ++n) {
                    long long r = 0;
                    for (int k = 0; k < KK; ++k) {
                        int a = as ? (int)A[m * KK + k] : (int)(uint8_t)A[m * KK + k];
                        int b = bs ? (int)B[k * N + n] : (int)(uint8_t)B[k * N + n];
                        r += a * b;
                    }
                    if (m == 0 && n == 0) r00 = r;
                    long long d = D[m * N + n] - r;
                    if (d < 0) d = -d;
                    if (d > maxerr) maxerr = d;
                }
            printf("i8 probe a_signed=%d b_signed=%d: max err %lld  D[0]=%d ref %lld\n", as, bs, maxerr, D[0], r00);
        }
    return 0;
}
