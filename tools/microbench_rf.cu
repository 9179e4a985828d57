// tools/microbench_rf.cu -- operand-form throughput on sm_100a: is the
// half rate of 3-source integer/DPX instructions a register-read limit?
// Each kind runs NCHAIN independent chains per thread; lane-ops/clk/SM.
// Kinds with two instructions per chain step report per-instruction rates.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb tools/microbench_rf.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define ITERS 4096
#define NCHAIN 8

struct P { uint32_t c1, c2, c3; };

template <int KIND>
__global__ void kern(int *out, const __grid_constant__ P p, uint32_t rb, uint32_t rc, long long *cycles)
{
    uint32_t x[NCHAIN], y[NCHAIN];
    const uint32_t b = rb + threadIdx.x, c = rc ^ threadIdx.x;
#pragma unroll
    for (int k = 0; k < NCHAIN; k++) { x[k] = threadIdx.x * (k + 1); y[k] = threadIdx.x * (k + 7); }
    long long t0 = clock64();
#pragma unroll 4
    for (int it = 0; it < ITERS; it++) {
#pragma unroll
        for (int k = 0; k < NCHAIN; k++) {
            if (KIND == 0) x[k] = __viaddmax_u16x2(x[k], b, c);                 // 3 regs
            if (KIND == 1) x[k] = __viaddmax_u16x2(x[k], p.c1, c);              // b from the constant bank
            if (KIND == 2) x[k] = __viaddmax_u16x2(x[k], 0xfffdfffdu, c);       // b immediate
            if (KIND == 3) x[k] = __vimax3_u16x2(x[k], b, c);                   // 3 regs
            if (KIND == 4) x[k] = __vimax3_u16x2(x[k], b, p.c1);                // c from the constant bank
            if (KIND == 5) asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(x[k]) : "r"(b), "r"(c));  // IMAD 3 regs
            if (KIND == 6) asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(x[k]) : "r"(b), "r"(p.c1));  // IMAD const addend
            if (KIND == 7) asm volatile("mad.lo.s32 %0, %0, 3, %1;" : "+r"(x[k]) : "r"(c));  // IMAD imm multiplier
            if (KIND == 8) x[k] = __byte_perm(x[k], b, c);                      // PRMT 3 regs
            if (KIND == 9) x[k] = __byte_perm(x[k], b, 0x5410);                 // PRMT imm selector
            if (KIND == 10) {  // IMAD (fma pipe) + VIADDMNMX (alu pipe), both 3 regs: shared limit?
                asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(y[k]) : "r"(b), "r"(c));
                x[k] = __viaddmax_u16x2(x[k], b, c);
            }
            if (KIND == 11) {  // IMAD const addend + VIADDMNMX const b
                asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(y[k]) : "r"(b), "r"(p.c2));
                x[k] = __viaddmax_u16x2(x[k], p.c1, c);
            }
            if (KIND == 12) {  // VIMNMX.U16x2 (2 regs, full rate) + IMAD 3 regs
                asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(y[k]) : "r"(b), "r"(c));
                x[k] = __vmaxu2(x[k], b);
            }
            if (KIND == 13) {  // IADD3-style add of a constant (alu?) + VIADDMNMX 3 regs
                asm volatile("add.s32 %0, %0, %1;" : "+r"(y[k]) : "r"(p.c2));
                x[k] = __viaddmax_u16x2(x[k], b, c);
            }
            if (KIND == 14) x[k] = __viaddmax_u16x2(x[k], x[k], c);             // two sources the same register
            if (KIND == 15) x[k] = __viaddmax_u16x2(x[k], x[(k + 3) % NCHAIN], x[(k + 5) % NCHAIN]);  // 3 distinct live regs
            if (KIND == 16) {  // both pipes, 3 distinct live regs each (no operand reuse)
                asm volatile("mad.lo.s32 %0, %1, %2, %3;" : "=r"(y[k]) : "r"(y[(k + 1) % NCHAIN]), "r"(x[(k + 2) % NCHAIN]), "r"(y[(k + 3) % NCHAIN]));
                x[k] = __viaddmax_u16x2(x[k], x[(k + 3) % NCHAIN], y[(k + 5) % NCHAIN]);
            }
            if (KIND == 17) {  // both pipes, operands reused (as 10) for comparison with 16
                asm volatile("mad.lo.s32 %0, %0, %1, %2;" : "+r"(y[k]) : "r"(b), "r"(c));
                x[k] = __viaddmax_u16x2(x[k], b, c);
            }
            if (KIND == 18) {  // VIMNMX.U16x2 (2 srcs) distinct live regs
                x[k] = __vmaxu2(x[(k + 1) % NCHAIN], x[(k + 4) % NCHAIN]) + 0u;
            }
        }
    }
    long long t1 = clock64();
    uint32_t s = 0;
#pragma unroll
    for (int k = 0; k < NCHAIN; k++) s ^= x[k] ^ y[k];
    out[blockIdx.x * blockDim.x + threadIdx.x] = (int)s;
    if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
}

template <int KIND>
void run(const char *name, int sms, int threads, int ninst)
{
    int grid = sms;
    int *out;
    long long *cyc;
    cudaMalloc(&out, sizeof(int) * grid * threads);
    cudaMalloc(&cyc, sizeof(long long) * grid);
    P p{0xfffdfffdu, 0xfffbfffbu, 7u};
    kern<KIND><<<grid, threads>>>(out, p, 5, 9, cyc);
    cudaDeviceSynchronize();
    kern<KIND><<<grid, threads>>>(out, p, 5, 9, cyc);
    cudaDeviceSynchronize();
    long long h[1024];
    cudaMemcpy(h, cyc, sizeof(long long) * grid, cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < grid; i++) mx = h[i] > mx ? h[i] : mx;
    const double ops = (double)threads * ITERS * NCHAIN * ninst;
    printf("%-40s threads=%4d  lane-instr/clk/SM=%7.2f\n", name, threads, ops / (double)mx);
    cudaFree(out);
    cudaFree(cyc);
}

int main()
{
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int th : {128, 256, 512}) {
        run<0>("VIADDMNMX.U16x2 r,r,r", sms, th, 1);
        run<1>("VIADDMNMX.U16x2 r,c,r", sms, th, 1);
        run<2>("VIADDMNMX.U16x2 r,imm,r", sms, th, 1);
        run<3>("VIMNMX3.U16x2 r,r,r", sms, th, 1);
        run<4>("VIMNMX3.U16x2 r,r,c", sms, th, 1);
        run<5>("IMAD r,r,r", sms, th, 1);
        run<6>("IMAD r,r,c", sms, th, 1);
        run<7>("IMAD r,imm,r", sms, th, 1);
        run<8>("PRMT r,r,r", sms, th, 1);
        run<9>("PRMT r,imm,r", sms, th, 1);
        run<10>("IMAD r,r,r + VIADDMNMX r,r,r", sms, th, 2);
        run<11>("IMAD r,r,c + VIADDMNMX r,c,r", sms, th, 2);
        run<12>("IMAD r,r,r + VIMNMX.U16x2 r,r", sms, th, 2);
        run<13>("IADD r,c + VIADDMNMX r,r,r", sms, th, 2);
        run<14>("VIADDMNMX.U16x2 x,x,r", sms, th, 1);
        run<15>("VIADDMNMX.U16x2 3 distinct live regs", sms, th, 1);
        run<16>("IMAD + VIADDMNMX, 3 distinct regs each", sms, th, 2);
        run<17>("IMAD + VIADDMNMX, reused operands", sms, th, 2);
        run<18>("VIMNMX.U16x2 2 distinct live regs", sms, th, 1);
    }
    return 0;
}
