// tools/microbench_int.cu -- measure sm_100a integer / DPX issue rates.
//
// Each kernel runs NCHAIN independent dependency chains per thread of one
// instruction kind, for ITERS iterations, on a full grid (148 SMs x many warps).
// Reports lane-ops per clock per SM (using clock64 on-device cycle counts) and
// Gops/s (using CUDA events).  The per-SM rate of the busiest pipe is the
// roofline denominator r_pipe.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb tools/microbench_int.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define ITERS 4096
#define NCHAIN 8

template <int KIND>
__global__ void kern(int *out, int a0, int b0, long long *cycles)
{
    int x[NCHAIN];
    const int b = b0 + threadIdx.x, c = a0 ^ threadIdx.x;
#pragma unroll
    for (int k = 0; k < NCHAIN; k++) x[k] = threadIdx.x * (k + 1);
    long long t0 = clock64();
#pragma unroll 4
    for (int it = 0; it < ITERS; it++) {
#pragma unroll
        for (int k = 0; k < NCHAIN; k++) {
            if (KIND == 0) x[k] = __viaddmax_s32(x[k], b, c);            // VIADDMNMX
            if (KIND == 1) x[k] = __viaddmax_s32_relu(x[k], b, c);       // VIADDMNMX.RELU
            if (KIND == 2) x[k] = __vimax3_s32_relu(x[k], b, c);         // VIMNMX3.RELU
            if (KIND == 3) asm volatile("max.s32 %0, %0, %1;" : "+r"(x[k]) : "r"(b));   // IMNMX
            if (KIND == 4) asm volatile("add.s32 %0, %0, %1;" : "+r"(x[k]) : "r"(b));   // IADD3
            if (KIND == 10) asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(x[k]) : "r"(b), "r"(c)); // IMAD
            if (KIND == 5) x[k] = __byte_perm(x[k], b, c);               // PRMT
            if (KIND == 6) x[k] = __vimax3_s32(x[k], b, c);              // VIMNMX3
            if (KIND == 7) x[k] = __viaddmax_s16x2(x[k], b, c);          // VIADDMNMX.S16x2
            if (KIND == 8) x[k] = __vimax3_s16x2_relu(x[k], b, c);       // VIMNMX3.S16x2.RELU
            if (KIND == 9) { x[k] = max(x[k] + b, c); }                   // IADD+IMNMX (compiler's choice)
            if (KIND == 11) x[k] = __vmaxu2(x[k], b);                      // VIMNMX.U16x2
            if (KIND == 12) x[k] = __vimax3_u16x2(x[k], b, c);            // VIMNMX3.U16x2
            if (KIND == 13) x[k] = __viaddmax_u16x2(x[k], b, c);          // VIADDMNMX.U16x2
        }
    }
    long long t1 = clock64();
    int s = 0;
#pragma unroll
    for (int k = 0; k < NCHAIN; k++) s ^= x[k];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
}

template <int KIND>
void run(const char *name, int sms, int threads, int ctas_per_sm)
{
    int grid = sms * ctas_per_sm;
    int *out;
    long long *cyc;
    cudaMalloc(&out, sizeof(int) * grid * threads);
    cudaMalloc(&cyc, sizeof(long long) * grid);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    kern<KIND><<<grid, threads>>>(out, 3, 5, cyc);
    cudaEventRecord(e0);
    const int reps = 5;
    for (int r = 0; r < reps; r++) kern<KIND><<<grid, threads>>>(out, 3, 5, cyc);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    long long *h = new long long[grid];
    cudaMemcpy(h, cyc, sizeof(long long) * grid, cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < grid; i++) mx = h[i] > mx ? h[i] : mx;
    double ops = (double)grid * threads * ITERS * NCHAIN;  // lane-ops per launch
    double per_sm_clk = ops / sms / (double)mx;             // lane-ops / clk / SM (in-kernel clock)
    double gops = ops * reps / (ms * 1e-3) / 1e9;
    printf("%-22s threads=%4d ctas/sm=%d  lane-ops/clk/SM=%7.2f  Gops/s=%9.1f  (max cyc %lld, %.3f ms/launch)\n",
           name, threads, ctas_per_sm, per_sm_clk, gops, mx, ms / reps);
    delete[] h;
    cudaFree(out);
    cudaFree(cyc);
}

int main()
{
    int dev = 0, sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    printf("SMs=%d clockRate(kHz)=%d\n", sms, clk);
    for (int thr : {256, 512, 1024}) {
        run<0>("VIADDMNMX", sms, thr, 1);
        run<1>("VIADDMNMX.RELU", sms, thr, 1);
        run<2>("VIMNMX3.RELU", sms, thr, 1);
        run<6>("VIMNMX3", sms, thr, 1);
        run<3>("IMNMX", sms, thr, 1);
        run<4>("IADD", sms, thr, 1);
        run<5>("PRMT", sms, thr, 1);
        run<7>("VIADDMNMX.S16x2", sms, thr, 1);
        run<8>("VIMNMX3.S16x2.RELU", sms, thr, 1);
        run<9>("IADD+IMNMX", sms, thr, 1);
        run<10>("IMAD", sms, thr, 1);
        run<11>("VIMNMX.U16x2", sms, thr, 1);
        run<12>("VIMNMX3.U16x2", sms, thr, 1);
        run<13>("VIADDMNMX.U16x2", sms, thr, 1);
    }
    return 0;
}
