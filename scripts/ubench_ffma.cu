// Micro-benchmark: FP32 FMA issue/pipe throughput per SM on sm_100a for the operand forms the layer
// kernels use (register, uniform-register/constant, immediate weight; FFMA vs packed FFMA2).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubf scripts/ubench_ffma.cu && /tmp/ubf
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kChains = 16;   // independent accumulators per thread
constexpr int kIters = 4096;  // loop trips, 32 FMAs per chain per trip

template <int FORM>
__global__ void kern(float* out, float w, float x0, long long* cycles) {
    float acc[kChains];
#pragma unroll
    for (int i = 0; i < kChains; ++i) acc[i] = x0 + i * 1e-3f + threadIdx.x * 1e-6f;
    float wr = w + threadIdx.x * 0.0f;  // a per-thread register copy (FORM 0)
    __syncthreads();
    long long t0 = clock64();
    for (int it = 0; it < kIters; ++it) {
#pragma unroll
        for (int k = 0; k < 32; ++k) {
#pragma unroll
            for (int i = 0; i < kChains; ++i) {
                if constexpr (FORM == 0) acc[i] = fmaf(acc[i], wr, acc[(i + 1) % kChains]);
                if constexpr (FORM == 1) acc[i] = fmaf(acc[i], w, acc[(i + 1) % kChains]);  // uniform / c-bank
                if constexpr (FORM == 2) acc[i] = fmaf(acc[i], 0.0625f, acc[(i + 1) % kChains]);  // immediate
            }
        }
        if constexpr (FORM == 3 || FORM == 4) {
        }
    }
    if constexpr (FORM == 3 || FORM == 4) {
        unsigned long long p[kChains / 2];
#pragma unroll
        for (int i = 0; i < kChains / 2; ++i)
            asm("mov.b64 %0, {%1, %2};" : "=l"(p[i]) : "f"(acc[2 * i]), "f"(acc[2 * i + 1]));
        unsigned long long W;
        const float wv = FORM == 3 ? w : 0.0625f;
        asm("mov.b64 %0, {%1, %2};" : "=l"(W) : "f"(wv), "f"(wv));
        for (int it = 0; it < kIters; ++it) {
#pragma unroll
            for (int k = 0; k < 32; ++k) {
#pragma unroll
                for (int i = 0; i < kChains / 2; ++i)
                    asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(p[i]) : "l"(W), "l"(p[(i + 1) % (kChains / 2)]));
            }
        }
#pragma unroll
        for (int i = 0; i < kChains / 2; ++i)
            asm("mov.b64 {%0, %1}, %2;" : "=f"(acc[2 * i]), "=f"(acc[2 * i + 1]) : "l"(p[i]));
    }
    long long t1 = clock64();
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < kChains; ++i) s += acc[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
}

template <int FORM>
void run(const char* name, int threads) {
    float* out;
    long long* cyc;
    const int blocks = 148;
    cudaMalloc(&out, sizeof(float) * blocks * threads);
    cudaMalloc(&cyc, sizeof(long long) * blocks);
    kern<FORM><<<blocks, threads>>>(out, 0.0625f, 1.0f, cyc);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<FORM><<<blocks, threads>>>(out, 0.0625f, 1.0f, cyc);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    long long c;
    cudaMemcpy(&c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
    const double fmas = (double)blocks * threads * kIters * 32 * kChains;
    const double per_sm_clk = (double)threads * kIters * 32 * kChains / (double)c;
    printf("%-28s threads %4d: %.1f TFMA/s, %.1f FMA/clk/SM (cycles %lld)\n", name, threads, fmas / ms / 1e9,
           per_sm_clk, c);
    cudaFree(out);
    cudaFree(cyc);
}

int main() {
    for (int th : {256, 512, 1024}) {
        run<0>("FFMA reg weight", th);
        run<1>("FFMA uniform weight", th);
        run<2>("FFMA immediate weight", th);
        run<3>("FFMA2 reg-pair weight", th);
        run<4>("FFMA2 imm-pair weight", th);
    }
    return 0;
}
