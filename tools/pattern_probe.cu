// Memory-pattern probe (no compute): copies a 2^n-amplitude complex64 state
// in place, tile by tile, with the same tile -> address map as the register-
// blocked passes (tile = 2^T amplitudes at the qubit positions S, runs of
// 2^r contiguous amplitudes), so its bandwidth is the HBM ceiling of a pass
// with that tile set.  Each CTA loads its whole tile into registers (16 B per
// thread and step), then stores it back.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/pattern_probe tools/pattern_probe.cu
//   tools/pattern_probe <n> "<S list>" ...
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <string>
#include <cuda_runtime.h>

struct Map {
    int nh;          // tile positions above the run
    int h[16];       // their qubits
    int nf;          // free qubit runs (tile index -> address)
    int fq[32], fl[32], fb[32];
};

__constant__ Map cm;

__device__ __forceinline__ unsigned long long tile_base(unsigned long long u) {
    unsigned long long a = 0;
    for (int i = 0; i < cm.nf; ++i) a |= ((u >> cm.fb[i]) & ((1ull << cm.fl[i]) - 1ull)) << cm.fq[i];
    return a;
}

__device__ __forceinline__ float4 ld256(const float4* p) {
    float4 v;
    asm volatile("ld.global.cs.L2::256B.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}

// mode 0: tile u = blockIdx + k grid; 1: same, loads with the L2::256B
// prefetch-size hint; 2: each CTA takes 2 consecutive tiles back to back
// (L2::256B); 3: 4 consecutive tiles (L2::256B)
template <int UPT, int mode>
__global__ void __launch_bounds__(512) probe(float4* psi, unsigned long long ntiles, int r) {
    // unit = 16 B = 2 amplitudes; tile = 256 threads * UPT units
    constexpr int gsh = mode == 2 ? 1 : mode == 3 ? 2 : 0;
    int lg = 0;
    while ((1ull << lg) < ntiles) ++lg;
    const unsigned long long per = (ntiles + gridDim.x - 1) / gridDim.x;
    for (unsigned long long k = blockIdx.x; (k << gsh) < ntiles; k += gridDim.x)
    for (unsigned long long u0 = k << gsh; u0 < ((k + 1) << gsh); ++u0) {
        // mode 4: CTA b takes tiles [b per, (b+1) per); 5: bit-reversed tile order
        unsigned long long u = u0;
        if (mode == 4) {
            const unsigned long long it = u0 / gridDim.x, b = u0 % gridDim.x;
            u = b * per + it;
            if (u >= ntiles) continue;
        } else if (mode == 5) {
            u = __brevll(u0) >> (64 - lg);
        }
        const unsigned long long base = tile_base(u);
        float4 v[UPT];
#pragma unroll
        for (int i = 0; i < UPT; ++i) {
            const unsigned t = 2u * (threadIdx.x + blockDim.x * i);  // tile index (amplitudes)
            unsigned long long g = t & ((1u << r) - 1u);
            const unsigned hi = t >> r;
            for (int b = 0; b < cm.nh; ++b)
                if ((hi >> b) & 1u) g += 1ull << cm.h[b];
            const float4* ptr = reinterpret_cast<float4*>(reinterpret_cast<float2*>(psi) + base + g);
            v[i] = mode ? ld256(ptr) : __ldcs(ptr);
        }
#pragma unroll
        for (int i = 0; i < UPT; ++i) {
            const unsigned t = 2u * (threadIdx.x + blockDim.x * i);
            unsigned long long g = t & ((1u << r) - 1u);
            const unsigned hi = t >> r;
            for (int b = 0; b < cm.nh; ++b)
                if ((hi >> b) & 1u) g += 1ull << cm.h[b];
            v[i].x += 0.f;
            __stcs(reinterpret_cast<float4*>(reinterpret_cast<float2*>(psi) + base + g), v[i]);
        }
    }
}

int main(int argc, char** argv) {
    const int n = atoi(argv[1]);
    float4* psi;
    const size_t bytes = 8ull << n;
    if (cudaMalloc(&psi, bytes) != cudaSuccess) return 1;
    cudaMemset(psi, 0, bytes);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    std::vector<std::string> specs;
    for (int a = 2; a < argc; ++a) {
        int cnt, seed, pin;
        if (sscanf(argv[a], "rand:%d:%d:%d", &cnt, &seed, &pin) == 3) {
            srand(seed);
            for (int c = 0; c < cnt; ++c) {
                std::vector<char> in(n, 0);
                for (int q = 0; q < pin; ++q) in[q] = 1;
                int have = pin;
                while (have < 13) {
                    const int q = pin + rand() % (n - pin);
                    if (!in[q]) in[q] = 1, ++have;
                }
                std::string sp;
                for (int q = 0; q < n; ++q)
                    if (in[q]) sp += (sp.empty() ? "" : ",") + std::to_string(q);
                specs.push_back(sp);
            }
        } else {
            specs.push_back(argv[a]);
        }
    }
    for (size_t a = 0; a < specs.size(); ++a) {
        std::vector<int> S;
        char name[256];
        snprintf(name, sizeof(name), "%s", specs[a].c_str());
        char buf[256];
        snprintf(buf, sizeof(buf), "%s", specs[a].c_str());
        for (char* p = strtok(buf, ","); p; p = strtok(nullptr, ",")) S.push_back(atoi(p));
        const int T = (int)S.size();
        int r = 0;
        while (r < T && S[r] == r) ++r;
        Map m{};
        m.nh = 0;
        for (int i = r; i < T; ++i) m.h[m.nh++] = S[i];
        std::vector<char> in(n, 0);
        for (int q : S) in[q] = 1;
        int b = 0;
        for (int q = 0; q < n;) {
            if (in[q]) { ++q; continue; }
            int e = q;
            while (e < n && !in[e]) ++e;
            m.fq[m.nf] = q; m.fl[m.nf] = e - q; m.fb[m.nf] = b; ++m.nf;
            b += e - q; q = e;
        }
        cudaMemcpyToSymbol(cm, &m, sizeof(m));
        const unsigned long long ntiles = 1ull << (n - T);
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0); cudaEventCreate(&e1);
        float best = 1e30f;
        for (int mode = 0; mode < 1; ++mode)
        for (int occ = 2; occ <= 2; occ *= 2) {
            for (int rep = 0; rep < 4; ++rep) {
                cudaEventRecord(e0);
                auto k = mode == 0 ? probe<16, 0> : mode == 1 ? probe<16, 4> : mode == 2 ? probe<16, 5> : probe<16, 1>;
                k<<<sms * (T >= 14 ? 1 : occ), 1u << (T - 5)>>>(psi, ntiles, r);
                cudaEventRecord(e1);
                cudaEventSynchronize(e1);
                float ms; cudaEventElapsedTime(&ms, e0, e1);
                if (rep) best = ms < best ? ms : best;
                if (rep == 3) printf("S=%s mode %d grid=%d*%d: %.3f ms = %.0f GB/s\n", name, mode, sms, occ, ms, 2.0 * bytes / ms / 1e6);
            }
        }
        if (cudaGetLastError() != cudaSuccess) { printf("error\n"); return 1; }
    }
    return 0;
}
