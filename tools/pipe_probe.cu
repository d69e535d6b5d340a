// Throughput probe of the FP32 FMA forms used by the apply kernels
// (FFMA with a uniform-register operand, 3-register FFMA, packed FFMA2 with
// a uniform pair).  usage: nvcc -arch=sm_100a -O3 pipe_probe.cu && ./a.out
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {
    unsigned long long d;
    asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d)
                 : "l"(*reinterpret_cast<unsigned long long*>(&a)), "l"(*reinterpret_cast<unsigned long long*>(&b)),
                   "l"(*reinterpret_cast<unsigned long long*>(&c)));
    return *reinterpret_cast<float2*>(&d);
}
constexpr int CH = 16, IT = 4096;
__global__ void k_ur(float* out, float m0, float m1) {  // FFMA R, R, UR, R
    float y[CH];
    for (int i = 0; i < CH; ++i) y[i] = threadIdx.x + i;
    for (int it = 0; it < IT; ++it)
#pragma unroll
        for (int i = 0; i < CH; ++i) y[i] = fmaf(y[i], m0, m1);
    float s = 0;
    for (int i = 0; i < CH; ++i) s += y[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_3r(float* out, float m0) {  // FFMA R, R, R, R
    float y[CH], z[CH];
    for (int i = 0; i < CH; ++i) { y[i] = threadIdx.x + i; z[i] = m0 * i; }
    for (int it = 0; it < IT; ++it)
#pragma unroll
        for (int i = 0; i < CH; ++i) y[i] = fmaf(y[i], z[i], z[(i + 1) % CH]);
    float s = 0;
    for (int i = 0; i < CH; ++i) s += y[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_f2(float* out, float m0, float m1) {  // FFMA2 R2, R2, UR2
    float2 y[CH];
    for (int i = 0; i < CH; ++i) y[i] = make_float2(threadIdx.x + i, i);
    const float2 mm = make_float2(m0, m1);
    for (int it = 0; it < IT; ++it)
#pragma unroll
        for (int i = 0; i < CH; ++i) y[i] = ffma2(y[i], mm, y[(i + 3) % CH]);
    float s = 0;
    for (int i = 0; i < CH; ++i) s += y[i].x + y[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_f2s(float* out, float m0, float m1) {  // FFMA2 R2, R2.swapped, UR2, R2 (complex MAC half)
    float2 y[CH], x[CH];
    for (int i = 0; i < CH; ++i) { y[i] = make_float2(threadIdx.x + i, i); x[i] = make_float2(i, -i); }
    const float2 mm = make_float2(-m0, m1);
    for (int it = 0; it < IT; ++it)
#pragma unroll
        for (int i = 0; i < CH; ++i) y[i] = ffma2(mm, make_float2(y[(i + 3) % CH].y, y[(i + 3) % CH].x), y[i]);
    float s = 0;
    for (int i = 0; i < CH; ++i) s += y[i].x + y[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
int main() {
    float* d;
    cudaMalloc(&d, 148 * 8 * 1024 * sizeof(float));
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int blocks = 148 * 8, thr = 256;
    const double insts = (double)blocks * thr / 32 * IT * CH;  // warp instructions
    for (int rep = 0; rep < 2; ++rep) {
        float ms;
        cudaEventRecord(a); k_ur<<<blocks, thr>>>(d, 1.0001f, 0.5f); cudaEventRecord(b); cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("FFMA R,R,UR,R   : %.3f warp-inst/clk/SM-sub @1.9GHz (%.2f ms)\n", insts / (ms * 1e-3) / (148 * 4) / 1.9e9, ms);
        cudaEventRecord(a); k_3r<<<blocks, thr>>>(d, 0.999f); cudaEventRecord(b); cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("FFMA R,R,R,R    : %.3f (%.2f ms)\n", insts / (ms * 1e-3) / (148 * 4) / 1.9e9, ms);
        cudaEventRecord(a); k_f2<<<blocks, thr>>>(d, 1.0001f, 0.999f); cudaEventRecord(b); cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("FFMA2 R2,R2,UR2  : %.3f (%.2f ms)\n", insts / (ms * 1e-3) / (148 * 4) / 1.9e9, ms);
        cudaEventRecord(a); k_f2s<<<blocks, thr>>>(d, 1.0001f, 0.999f); cudaEventRecord(b); cudaEventSynchronize(b);
        cudaEventElapsedTime(&ms, a, b);
        printf("FFMA2 swapped    : %.3f (%.2f ms)\n", insts / (ms * 1e-3) / (148 * 4) / 1.9e9, ms);
    }
    return 0;
}
