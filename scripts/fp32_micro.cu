// Micro-benchmark of FP32-pipe issue rates on B200 (for the k-means roofline in DESIGN.md):
// scalar FFMA (3 registers), packed FFMA2 / FADD2, and the FADD2+FFMA2 pair the k-means
// distance uses. Each thread runs 8 independent dependency chains; prints lane-ops/s.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp32_micro fp32_micro.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kIters = 4096;

__global__ void k_ffma(float* out, float a, float b) {
    float x[8];
    for (int i = 0; i < 8; ++i) x[i] = threadIdx.x * 0.001f + i;
    for (int it = 0; it < kIters; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) x[i] = __fmaf_rn(x[i], a, b);
    float s = 0;
    for (int i = 0; i < 8; ++i) s += x[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_ffma2(float* out, float a, float b) {
    float2 x[8];
    for (int i = 0; i < 8; ++i) x[i] = make_float2(threadIdx.x * 0.001f + i, i);
    const float2 aa = make_float2(a, a + 1), bb = make_float2(b, b + 1);
    for (int it = 0; it < kIters; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) x[i] = __ffma2_rn(x[i], aa, bb);
    float s = 0;
    for (int i = 0; i < 8; ++i) s += x[i].x + x[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_fadd2(float* out, float a, float b) {
    float2 x[8];
    for (int i = 0; i < 8; ++i) x[i] = make_float2(threadIdx.x * 0.001f + i, i);
    const float2 aa = make_float2(a, b);
    for (int it = 0; it < kIters; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) x[i] = __fadd2_rn(x[i], aa);
    float s = 0;
    for (int i = 0; i < 8; ++i) s += x[i].x + x[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// the k-means inner step: d = x + (-c); acc = fma(d, d, acc), packed. The add's operand is the
// running accumulator so the compiler cannot hoist it out of the loop (an earlier version added
// two loop invariants, the FADD2 was hoisted and the pair was counted at twice its real rate).
__global__ void k_pair(float* out, float a, float b) {
    float2 acc[8];
    for (int i = 0; i < 8; ++i) acc[i] = make_float2(threadIdx.x * 1e-9f, i * 1e-9f);
    const float2 nc = make_float2(-a * 1e-6f, -b * 1e-6f);
    for (int it = 0; it < kIters; ++it)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const float2 d = __fadd2_rn(acc[i], nc);
            acc[i] = __ffma2_rn(d, d, acc[i]);
        }
    float s = 0;
    for (int i = 0; i < 8; ++i) s += acc[i].x + acc[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <typename K>
double run(K kern, const char* name, double lane_ops_per_thread_iter, int blocks, int threads, float* out) {
    kern<<<blocks, threads>>>(out, 1.0001f, 0.5f);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    for (int r = 0; r < 5; ++r) kern<<<blocks, threads>>>(out, 1.0001f, 0.5f);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    const double ops = 5.0 * blocks * threads * (double)kIters * lane_ops_per_thread_iter;
    const double r = ops / (ms / 1e3);
    printf("{\"kernel\": \"%s\", \"blocks\": %d, \"threads\": %d, \"lane_ops_per_s\": %.4e}\n", name, blocks, threads, r);
    return r;
}

int main() {
    int sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    printf("{\"sms\": %d, \"clock_khz\": %d}\n", sms, clk);
    float* out;
    cudaMalloc(&out, sizeof(float) * 148 * 8 * 1024);
    for (int bpsm : {4, 8}) {
        run(k_ffma, "ffma_3reg", 8, sms * bpsm, 256, out);
        run(k_ffma2, "ffma2", 16, sms * bpsm, 256, out);
        run(k_fadd2, "fadd2", 16, sms * bpsm, 256, out);
        run(k_pair, "fadd2+ffma2", 32, sms * bpsm, 256, out);
    }
    return 0;
}
