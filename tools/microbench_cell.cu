// tools/microbench_cell.cu -- throughput of alternative SW/Gotoh cell-update
// formulations on sm_100a (registers only, ALPHA rows x 2 columns per step,
// the same dependency structure as sw_fill.cuh).  Reports cells/clk/SM.
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mbc tools/microbench_cell.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define ALPHA 16
#define STEPS 2048

__device__ __forceinline__ int prmt(uint32_t a, uint32_t b, uint32_t sel)
{
    int r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
    return r;
}
// add through the FMA pipe: x * one + y with `one` unknown to the compiler
__device__ __forceinline__ int imad(int x, int one, int y)
{
    int r;
    asm("mad.lo.s32 %0, %1, %2, %3;" : "=r"(r) : "r"(x), "r"(one), "r"(y));
    return r;
}

template <int F>
__global__ void kern(int *out, const uint32_t *prof, const uint32_t *sels, int ge, int gf, int one, long long *cyc)
{
    uint32_t P[ALPHA];
    int e[ALPHA], t[ALPHA];
#pragma unroll
    for (int r = 0; r < ALPHA; r++) {
        P[r] = prof[(threadIdx.x + r) & 15];
        e[r] = -1000;
        t[r] = -gf;
    }
    int tprev = -gf, ot0 = 0, of0 = -1000, ot1 = 0, of1 = -1000, tmax = 0;
    const int nge = -ge;
    long long c0 = clock64();
    for (int k = 0; k < STEPS; k++) {
        int a_t = __shfl_up_sync(0xffffffffu, ot0, 1);
        int a_f = __shfl_up_sync(0xffffffffu, of0, 1);
        int b_t = __shfl_up_sync(0xffffffffu, ot1, 1);
        int b_f = __shfl_up_sync(0xffffffffu, of1, 1);
        const uint2 sl = make_uint2(sels[k & 63], sels[(k + 1) & 63]);
        int tdA = tprev, tdB = a_t;
        tprev = b_t;
        int tuA = a_t, fuA = a_f, tuB = b_t, fuB = b_f;
#pragma unroll
        for (int r = 0; r < ALPHA; r++) {
            int eA, hA, eB, hB;
            if (F == 0) {  // current kernel
                eA = __viaddmax_s32(e[r], nge, t[r]);
                fuA = max(fuA - ge, tuA);
                int pA = prmt(P[r], 0x80808080u, sl.x);
                hA = __viaddmax_s32_relu(tdA, pA, max(eA, fuA));
            } else if (F == 1) {  // adds on the FMA pipe, plain max on ALU
                eA = max(imad(e[r], one, nge), t[r]);
                fuA = max(imad(fuA, one, nge), tuA);
                int pA = prmt(P[r], 0x80808080u, sl.x);
                hA = __vimax3_s32_relu(eA, fuA, imad(tdA, one, pA));
            } else if (F == 2) {  // E DPX, F on FMA+max, H vimax3.relu
                eA = __viaddmax_s32(e[r], nge, t[r]);
                fuA = max(imad(fuA, one, nge), tuA);
                int pA = prmt(P[r], 0x80808080u, sl.x);
                hA = __vimax3_s32_relu(eA, fuA, imad(tdA, one, pA));
            } else {  // E/F on FMA+max, H DPX relu
                eA = max(imad(e[r], one, nge), t[r]);
                fuA = max(imad(fuA, one, nge), tuA);
                int pA = prmt(P[r], 0x80808080u, sl.x);
                hA = __viaddmax_s32_relu(tdA, pA, max(eA, fuA));
            }
            tdA = t[r];
            const int tA = (F == 0) ? hA - gf : imad(hA, one, -gf);
            tuA = tA;
            if (F == 0) {
                eB = __viaddmax_s32(eA, nge, tA);
                fuB = max(fuB - ge, tuB);
                int pB = prmt(P[r], 0x80808080u, sl.y);
                hB = __viaddmax_s32_relu(tdB, pB, max(eB, fuB));
            } else if (F == 1) {
                eB = max(imad(eA, one, nge), tA);
                fuB = max(imad(fuB, one, nge), tuB);
                int pB = prmt(P[r], 0x80808080u, sl.y);
                hB = __vimax3_s32_relu(eB, fuB, imad(tdB, one, pB));
            } else if (F == 2) {
                eB = __viaddmax_s32(eA, nge, tA);
                fuB = max(imad(fuB, one, nge), tuB);
                int pB = prmt(P[r], 0x80808080u, sl.y);
                hB = __vimax3_s32_relu(eB, fuB, imad(tdB, one, pB));
            } else {
                eB = max(imad(eA, one, nge), tA);
                fuB = max(imad(fuB, one, nge), tuB);
                int pB = prmt(P[r], 0x80808080u, sl.y);
                hB = __viaddmax_s32_relu(tdB, pB, max(eB, fuB));
            }
            tdB = tA;
            const int tB = (F == 0) ? hB - gf : imad(hB, one, -gf);
            tuB = tB;
            e[r] = eB;
            t[r] = tB;
            tmax = __vimax3_s32(tmax, hA, hB);
        }
        ot0 = tuA; of0 = fuA; ot1 = tuB; of1 = fuB;
    }
    long long c1 = clock64();
    int s = tmax ^ ot0 ^ of1;
#pragma unroll
    for (int r = 0; r < ALPHA; r++) s ^= e[r] + t[r];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
}

// Packed 16x2: each 32-bit register holds (row i, col j) and (row i+8, col j-1)
// as biased unsigned 16-bit values; adds via IMAD (carry-free: halves stay in
// [0, 65535]), maxima via VIMNMX(3).U16x2.  8 packed slots = 16 rows.
template <int F>
__global__ void kernp(int *out, const uint32_t *prof, const uint32_t *sels, int ge, int gf, int one, long long *cyc)
{
    uint32_t P[8], Q[8];
    uint32_t e[8], t[8];
    const uint32_t nge2 = (uint32_t)(0x10000 - ge) * 0x10001u;  // unused (adds of negatives avoided)
    (void)nge2;
    const uint32_t ge2 = (uint32_t)ge * 0x10001u, gf2 = (uint32_t)gf * 0x10001u, fl2 = 0x40004000u;
#pragma unroll
    for (int r = 0; r < 8; r++) {
        P[r] = prof[(threadIdx.x + r) & 15];
        Q[r] = prof[(threadIdx.x + r + 8) & 15];
        e[r] = 0x40004000u;
        t[r] = 0x40004000u;
    }
    uint32_t tprev = 0x40004000u, ot = 0x40004000u, of = 0x40004000u, tmax = 0;
    long long c0 = clock64();
    for (int k = 0; k < STEPS; k++) {
        uint32_t up_t = __shfl_up_sync(0xffffffffu, ot, 1);
        uint32_t up_f = __shfl_up_sync(0xffffffffu, of, 1);
        const uint32_t sel = sels[k & 63];
        // slot-0 inputs: lo half = upper lane's hi half, hi half = own slot-7 lo half
        uint32_t tu = __byte_perm(up_t, t[7], 0x5432);
        uint32_t fu = __byte_perm(up_f, of, 0x5432);
        uint32_t td = tprev;
        tprev = tu;
#pragma unroll
        for (int r = 0; r < 8; r++) {
            // E: a = max(e - ge, t_left)
            uint32_t ea = __vmaxu2(e[r] - ge2, t[r]);
            // F: max(fu - ge, tu)
            fu = __vmaxu2(fu - ge2, tu);
            uint32_t p = prmt(P[r], Q[r], sel);
            uint32_t x = (uint32_t)imad((int)td, one, (int)p);
            uint32_t h = __vimax3_u16x2(ea, fu, x);
            if (F == 1) h = __vmaxu2(h, fl2);
            td = t[r];
            uint32_t tt = (uint32_t)imad((int)h, one, -(int)gf2);
            tu = tt;
            e[r] = ea;
            t[r] = tt;
            if (r & 1) tmax = __vimax3_u16x2(tmax, h, tt);
        }
        ot = tu;
        of = fu;
    }
    long long c1 = clock64();
    uint32_t s = tmax ^ ot ^ of;
#pragma unroll
    for (int r = 0; r < 8; r++) s ^= e[r] + t[r];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
}

template <int F>
void runp(int sms, int threads, int ctas, const uint32_t *prof, const uint32_t *sels)
{
    int grid = sms * ctas;
    int *out;
    long long *cyc;
    cudaMalloc(&out, sizeof(int) * grid * threads);
    cudaMalloc(&cyc, sizeof(long long) * grid);
    kernp<F><<<grid, threads>>>(out, prof, sels, 2, 5, 1, cyc);
    cudaDeviceSynchronize();
    kernp<F><<<grid, threads>>>(out, prof, sels, 2, 5, 1, cyc);
    cudaDeviceSynchronize();
    long long *h = new long long[grid];
    cudaMemcpy(h, cyc, sizeof(long long) * grid, cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < grid; i++) mx = h[i] > mx ? h[i] : mx;
    double cells = (double)grid * threads * STEPS * 16;
    printf("P%d threads=%4d ctas/sm=%d  cells/clk/SM=%6.2f\n", F, threads, ctas, cells / sms / mx);
    delete[] h;
    cudaFree(out);
    cudaFree(cyc);
}

template <int F>
void run(int sms, int threads, int ctas, const uint32_t *prof, const uint32_t *sels)
{
    int grid = sms * ctas;
    int *out;
    long long *cyc;
    cudaMalloc(&out, sizeof(int) * grid * threads);
    cudaMalloc(&cyc, sizeof(long long) * grid);
    kern<F><<<grid, threads>>>(out, prof, sels, 2, 5, 1, cyc);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<F><<<grid, threads>>>(out, prof, sels, 2, 5, 1, cyc);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    long long *h = new long long[grid];
    cudaMemcpy(h, cyc, sizeof(long long) * grid, cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < grid; i++) mx = h[i] > mx ? h[i] : mx;
    double cells = (double)grid * threads * STEPS * 2 * ALPHA;
    printf("F%d threads=%4d ctas/sm=%d  cells/clk/SM=%6.2f  GCUPS=%8.1f\n", F, threads, ctas, cells / sms / mx,
           cells / (ms * 1e-3) / 1e9);
    delete[] h;
    cudaFree(out);
    cudaFree(cyc);
}

int main()
{
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    uint32_t hp[16]; for (int i = 0; i < 16; i++) { const uint32_t b[4] = {0x02020206u, 0x02020602u, 0x02060202u, 0x06020202u}; hp[i] = b[i & 3]; }
    uint32_t hs[64];
    for (int i = 0; i < 64; i++) {
        uint32_t c = (i * 7 + 3) & 3, s = c | 8;
        hs[i] = c | (s << 4) | (s << 8) | (s << 12);
    }
    uint32_t *prof, *sels;
    cudaMalloc(&prof, sizeof(hp));
    cudaMalloc(&sels, sizeof(hs));
    cudaMemcpy(prof, hp, sizeof(hp), cudaMemcpyHostToDevice);
    cudaMemcpy(sels, hs, sizeof(hs), cudaMemcpyHostToDevice);
    for (int w : {128, 256, 384, 512}) {
        run<0>(sms, w, 1, prof, sels);
        run<1>(sms, w, 1, prof, sels);
        run<2>(sms, w, 1, prof, sels);
        run<3>(sms, w, 1, prof, sels);
        runp<0>(sms, w, 1, prof, sels);
        runp<1>(sms, w, 1, prof, sels);
    }
    return 0;
}
