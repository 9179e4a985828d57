// sw_mm.cuh -- Stages 3-5 on the GPU (CUDAlign 2.0,
// Sandes & de Melo IPDPS 2011, P:<line> = /root/reference/PAPER.md line).
//
// Input: the crosspoint list L_2 of Stage 2, i.e. partitions
// (C_s, C_e) whose optimal score S = score_e - score_s is known.
// Output: the optimal alignment of every partition, concatenated into the
// full alignment.
//
// B200 design:
//  * Myers-Miller with balanced splitting and goal-based matching:
//    a partition larger than MM_TB_CELLS is split across its larger dimension
//    (rows, or columns by running the transposed problem): a forward global
//    pass from C_s to the middle line and a reverse pass from C_e to it, then
//    the junction of the two on that line: H_f + H_r = S, or for a gap that
//    crosses the line F_f + F_r + G_open = S (reading S18).  The new crosspoint
//    carries its type, so each half starts / ends in the right gap state
//    (P:160-162).  ONE WARP per partition; all partitions of a level in one
//    launch (they are independent).
//  * Stage 5: partitions at most MM_TB_CELLS cells get a full DP with
//    4-bit traceback codes in global memory (L2-resident) and one lane walks
//    them back; one warp per partition, one launch for all.
//
// The warp DP engine: lane = MM_ALPHA consecutive rows with H and E in
// registers, lanes skewed by one column (the row above comes by SHFL), chunks
// of 32 * MM_ALPHA rows run one after the other through a per-partition row
// buffer in global memory (lane 0 reads it through a 32-column prefetch,
// lane 31 writes the chunk's bottom row back in place).  All int32; the
// global recurrence has no 0 term.
#pragma once
#include <type_traits>
#include "sw_fill.cuh"

namespace swb {

#ifndef SWB_MM_ALPHA
#define SWB_MM_ALPHA 16
#endif
constexpr int MM_ALPHA = SWB_MM_ALPHA;  // rows per lane (a multiple of 8: one traceback word per 8 rows)
static_assert(MM_ALPHA % 8 == 0, "MM_ALPHA rows per lane: whole 8-row traceback words");
constexpr int MM_CHUNK = 32 * MM_ALPHA;
constexpr long long MM_TB_CELLS = 1 << 16;  // Stage-5 partitions: at most this many cells

struct MMPart {
    int i_s, j_s, i_e, j_e;  // DP cells of C_s and C_e (original coordinates)
    int t_s, t_e;            // crosspoint types: 0 pair / any, 1 gap in S0 (horizontal), 2 gap in S1 (vertical)
    int score;               // S(C_s, C_e) = score_e - score_s
    int pad;
    long long off;           // scratch offset (int2): split row buffer + two captured lines; Stage 5 row buffer
    long long off_c;         // Stage 5: traceback codes offset (u32)
    long long off_m;         // Stage 5: moves offset (bytes); the slice holds h + w bytes
};

struct MMRes {
    int i, j, type, sub;     // split crosspoint X and S(C_s, X); type -1: no junction found
};

struct MMArgs {
    const unsigned char *A, *B;  // ASCII S0, S1 (0-based; DP row i pairs A[i - 1])
    int ma, mi, go, ge, gf;
    uint32_t prof[4];    // row code a -> int8x4 word, byte x = (a == x ? ma : mi) + G_first
    int wide;            // 1: |p + G_first| > 127; p + G_first selected from pm_gf / pn_gf by comparing codes
    int pm_gf, pn_gf;
    int nparts;
    const MMPart *parts;
    int2 *scratch;
    MMRes *res;
    unsigned int *codes;
    char *moves;
    int *nmoves;
    int *err;            // set to 2 when a spin-wait times out (watchdog)
    int *cnt;            // CTA split kernel: passes finished per partition (zeroed per launch)
    long long timeout_ns;
};

// A global DP problem of h x w cells: row a (1..h) pairs rs[a * rstep],
// column b (1..w) pairs cs[b * cstep].  kind = boundary:
//   0 fresh start, 1 start inside a horizontal gap, 2 inside a vertical gap,
//   3 reverse pass from an end inside a vertical gap (leave it vertically),
//   4 reverse pass from an end inside a horizontal gap.
struct DpProb {
    const unsigned char *rs;
    const unsigned char *cs;
    int rstep, cstep;
    int h, w, kind;
};

__device__ __forceinline__ int mm_row0(const MMArgs &g, int kind, int b)  // H(0,b) = E(0,b), b >= 1
{
    if (kind == 3) return NEG;
    return kind == 1 ? -(b * g.ge) : -(g.go + b * g.ge);
}
__device__ __forceinline__ int mm_col0(const MMArgs &g, int kind, int a)  // H(a,0) = F(a,0), a >= 1
{
    if (kind == 4) return NEG;
    return kind == 2 ? -(a * g.ge) : -(g.go + a * g.ge);
}
__device__ __forceinline__ int mm_up(unsigned char c) { return c & 0xDF; }  // ASCII upper case (ACGT only)

// 2-bit code of an ASCII base, case-insensitive: A/a 0, C/c 1, T/t 2, G/g 3.
__device__ __forceinline__ uint32_t mm_code(unsigned char c) { return (c >> 1) & 3u; }

// One chunk of MM_CHUNK rows starting at row a0 + 1, swept over columns 1..w.
// The row above comes from rin (H, F per column; lane 0 reads it through a
// 32-column prefetch), the chunk's bottom row goes to rout (lane 31).  Lane
// state: rows r0+1 .. r0+MM_ALPHA as t = H - G_first and E, the substitution
// score p + G_first from an int8x4 profile word and one PRMT per cell (as the
// band kernel): per cell E = max(E - G_ext, t_left), F = max(F_up - G_ext, t_up),
// H = max(E, F, t_diag + (p + G_first)) (Eq. 1-3, no 0 term), t = H - G_first.
//   MODE 0: H, F of row capR into cap[b].
//   MODE 1: 4-bit traceback codes: bits 0-1 H source (0 diagonal, 1 F, 2 E;
//     ties prefer that order), bit 2 E extends (E(a,b-1) - G_ext >= t(a,b-1)),
//     bit 3 F extends; codes[b * HW + (a - 1) / 8], nibble (a - 1) % 8.
// wait(need): block until rin holds columns 1..need (CTA pipeline; no-op for
// one warp); publish(cols): rout holds columns 1..cols.
template <int MODE, bool CAPC, bool WIDE, class Wait, class Publish>
__device__ __forceinline__ void mm_chunk_impl(const MMArgs &g, const DpProb &P, int a0, const int2 *rin, int2 *rout,
                                              int capR, int2 *cap, unsigned int *codes, int lane, Wait wait,
                                              Publish publish)
{
    const int h = P.h, w = P.w, kind = P.kind;
    const int HW = (h + 7) / 8;
    const int gf = g.gf, nge = -g.ge;
    const int r0 = a0 + lane * MM_ALPHA;  // this lane: rows r0 + 1 .. r0 + MM_ALPHA
    uint32_t Pw[MM_ALPHA];
    int T[MM_ALPHA], E[MM_ALPHA];
#pragma unroll
    for (int r = 0; r < MM_ALPHA; r++) {
        const int a = r0 + r + 1;
        if constexpr (WIDE) Pw[r] = a <= h ? mm_code(P.rs[(long long)a * P.rstep]) : 5u;  // pad rows: never a match
        else Pw[r] = a <= h ? g.prof[mm_code(P.rs[(long long)a * P.rstep])] : PADPROF;
        T[r] = mm_col0(g, kind, a) - gf;
        E[r] = NEG;
    }
    const int diag00 = (kind == 3 || kind == 4) ? NEG : 0;
    int tdiag = (r0 == 0 ? diag00 : mm_col0(g, kind, r0)) - gf;  // t(r0, b - 1)
    int tu_out = 0, fu_out = 0;
    const bool cap_lane = CAPC && capR > r0 && capR <= r0 + MM_ALPHA;  // CAPC: this chunk holds row capR
    wait(64);
    int2 cur = (1 + lane <= w) ? __ldcg(rin + 1 + lane) : make_int2(NEG, NEG);
    int2 nxt = (33 + lane <= w) ? __ldcg(rin + 33 + lane) : make_int2(NEG, NEG);
    const int nsteps = w + 31;
    // column b's code (pad: never a match / the PADPROF byte), loaded one step
    // ahead so the byte load is off the step's dependency chain
    auto col_code = [&](int b) -> uint32_t {
        return (b >= 1 && b <= w) ? mm_code(__ldg(P.cs + (long long)b * P.cstep)) : (WIDE ? 6u : 4u);
    };
    uint32_t ccode = col_code(1 - lane);
    // GUARD (compile time): some lane is outside columns 1..w; those lanes compute
    // and discard (no early return: the warp stays converged for the shuffles)
    auto step = [&](int k, auto guard_c) {
        constexpr bool GUARD = decltype(guard_c)::value;
        int tu = __shfl_up_sync(0xffffffffu, tu_out, 1);
        int fu = __shfl_up_sync(0xffffffffu, fu_out, 1);
        const int rH = __shfl_sync(0xffffffffu, cur.x, k & 31);
        const int rF = __shfl_sync(0xffffffffu, cur.y, k & 31);
        if (lane == 0) { tu = rH - gf; fu = rF; }
        const int b = k - lane + 1;
        const bool ok = !GUARD || (b >= 1 && b <= w);
        const uint32_t code = ccode;
        ccode = col_code(b + 1);
        const uint32_t sel = WIDE ? code : code * 0x1111u + 0x8880u;  // col_sel(code)
        int td = tdiag;
        const int tu_in = tu;  // t(r0, b): the next step's diagonal
        int Tn[MM_ALPHA], En[MM_ALPHA];
        unsigned int tb[MM_ALPHA / 8] = {};
        int capH = 0, capF = 0;
#pragma unroll
        for (int r = 0; r < MM_ALPHA; r++) {
            const int e = __viaddmax_s32(E[r], nge, T[r]);   // Eq. 2
            const int f = __viaddmax_s32(fu, nge, tu);       // Eq. 3
            const int x = td + (WIDE ? (Pw[r] == sel ? g.pm_gf : g.pn_gf) : prmt(Pw[r], PADPROF, sel));  // H_diag + p
            const int hv = __vimax3_s32(e, f, x);            // Eq. 1 (global: no 0 term)
            if (MODE == 1) {
                const unsigned int src = (x >= e && x >= f) ? 0u : (f >= e ? 1u : 2u);
                const unsigned int ext = (E[r] + nge >= T[r] ? 4u : 0u) | (fu + nge >= tu ? 8u : 0u);
                tb[r / 8] |= (src | ext) << (4 * (r % 8));
            }
            if (CAPC && cap_lane && r0 + r + 1 == capR) { capH = hv; capF = f; }
            td = T[r];
            Tn[r] = hv - gf;
            En[r] = e;
            tu = Tn[r];
            fu = f;
        }
        tdiag = ok ? tu_in : tdiag;
#pragma unroll
        for (int r = 0; r < MM_ALPHA; r++) {
            T[r] = ok ? Tn[r] : T[r];
            E[r] = ok ? En[r] : E[r];
        }
        if (ok) {
            tu_out = tu;
            fu_out = fu;
            if (MODE == 1) {
#pragma unroll
                for (int q = 0; q < MM_ALPHA / 8; q++)
                    if (r0 + 8 * q < h) codes[(long long)b * HW + r0 / 8 + q] = tb[q];
            }
            if (CAPC && cap_lane) cap[b] = make_int2(capH, capF);
            if (lane == 31) rout[b] = make_int2(tu + gf, fu);
        }
    };
    for (int kb = 0; kb < nsteps; kb += 32) {
        if (kb > 0) {
            cur = nxt;
            wait(kb + 64);
            const int c = kb + 33 + lane;
            nxt = c <= w ? __ldcg(rin + c) : make_int2(NEG, NEG);
        }
        if (kb >= 32 && kb + 32 <= w) {
#pragma unroll 4
            for (int u = 0; u < 32; u++) step(kb + u, std::false_type{});
        } else {
            const int ke = min(kb + 32, nsteps);
#pragma unroll 1
            for (int k = kb; k < ke; k++) step(k, std::true_type{});
        }
        publish(min(w, kb + 1));
    }
}

// The int8-profile or the WIDE cell update (a uniform branch outside the cell loop).
template <int MODE, bool CAPC, class Wait, class Publish>
__device__ __forceinline__ void mm_chunk(const MMArgs &g, const DpProb &P, int a0, const int2 *rin, int2 *rout,
                                         int capR, int2 *cap, unsigned int *codes, int lane, Wait wait,
                                         Publish publish)
{
    if (g.wide) mm_chunk_impl<MODE, CAPC, true>(g, P, a0, rin, rout, capR, cap, codes, lane, wait, publish);
    else mm_chunk_impl<MODE, CAPC, false>(g, P, a0, rin, rout, capR, cap, codes, lane, wait, publish);
}

// One warp runs the whole pass (chunks one after the other, row buffer in place).
// MODE 0: rows 1..capR, H and F of row capR into cap (columns 0..w).
// MODE 1: all rows, traceback codes.
template <int MODE>
__device__ void mm_warp_dp(const MMArgs &g, const DpProb &P, int2 *rowbuf, int capR, int2 *cap, unsigned int *codes,
                           int lane)
{
    const int w = P.w, kind = P.kind;
    const int rows = MODE == 0 ? capR : P.h;
    for (int b = lane; b <= w; b += 32) {
        const int2 v = make_int2(b == 0 ? 0 : mm_row0(g, kind, b), (b == 0 && kind == 2) ? 0 : NEG);
        rowbuf[b] = v;
        if (MODE == 0 && capR == 0) cap[b] = v;
    }
    if (MODE == 0 && capR > 0 && lane == 0) cap[0] = make_int2(mm_col0(g, kind, capR), mm_col0(g, kind, capR));
    __threadfence_block();
    __syncwarp();
    for (int a0 = 0; a0 < rows; a0 += MM_CHUNK) {
        if (MODE == 0 && a0 + MM_CHUNK >= capR)
            mm_chunk<MODE, true>(g, P, a0, rowbuf, rowbuf, capR, cap, codes, lane, [](int) {}, [](int) {});
        else
            mm_chunk<MODE, false>(g, P, a0, rowbuf, rowbuf, capR, cap, codes, lane, [](int) {}, [](int) {});
        __threadfence_block();
        __syncwarp();
    }
}

// CTA version of the MODE-0 pass for large partitions: the NWP warps take the
// 256-row chunks round robin (chunk c on warp c % NWP).  Chunk c reads its top
// row from ring slot c % (NWP+1), written by chunk c-1, and writes its bottom
// row to slot (c+1) % (NWP+1); the writer publishes (generation, columns) in
// shared memory every 32 columns (after __threadfence_block), the reader's
// lane 0 waits for it before each 32-column prefetch and loads through L2
// (__ldcg).  A slot is reused by the same warp NWP chunks later, after its
// reader (the next warp) is done with it.
template <int NWP>
__device__ void mm_cta_pass(const MMArgs &g, const DpProb &P, int2 *ring, long long rs, int capR, int2 *cap,
                            volatile int *s_gen, volatile int *s_cols, int warp, int lane)
{
    constexpr int R = NWP + 1;
    const int w = P.w, kind = P.kind;
    for (int b = threadIdx.x; b <= w; b += blockDim.x) {
        const int2 v = make_int2(b == 0 ? 0 : mm_row0(g, kind, b), (b == 0 && kind == 2) ? 0 : NEG);
        ring[b] = v;
        if (capR == 0) cap[b] = v;
    }
    if (threadIdx.x < R) {
        s_gen[threadIdx.x] = threadIdx.x == 0 ? -1 : -2;
        s_cols[threadIdx.x] = threadIdx.x == 0 ? w : 0;
    }
    if (capR > 0 && threadIdx.x == 0) cap[0] = make_int2(mm_col0(g, kind, capR), mm_col0(g, kind, capR));
    __syncthreads();
    const int nchunks = (capR + MM_CHUNK - 1) / MM_CHUNK;
    for (int c = warp; c < nchunks; c += NWP) {
        const int in = c % R, out = (c + 1) % R;
        if (lane == 0) s_cols[out] = 0;
        __threadfence_block();
        if (lane == 0) s_gen[out] = c;
        __syncwarp();
        // every lane polls and the warp votes: the loop is warp-uniform, so the
        // warp stays converged for the cell loop's shuffles (a lane-0 spin made
        // ptxas route every step through its divergent-warp path)
        auto wait = [&](int need) {
            need = min(need, w);
            if (__any_sync(0xffffffffu, s_gen[in] != c - 1 || s_cols[in] < need)) {
                const unsigned long long t0 = gtimer();
                while (__any_sync(0xffffffffu, s_gen[in] != c - 1 || s_cols[in] < need)) {
                    __nanosleep(32);
                    if (__any_sync(0xffffffffu, gtimer() - t0 > (unsigned long long)g.timeout_ns)) {
                        if (lane == 0) atomicExch(g.err, 2);
                        break;
                    }
                }
            }
            __threadfence_block();
        };
        auto publish = [&](int cols) {
            __threadfence_block();
            __syncwarp();
            if (lane == 31) s_cols[out] = cols;
        };
        if ((c + 1) * MM_CHUNK >= capR)
            mm_chunk<0, true>(g, P, c * MM_CHUNK, ring + in * rs, ring + out * rs, capR, cap, nullptr, lane, wait, publish);
        else
            mm_chunk<0, false>(g, P, c * MM_CHUNK, ring + in * rs, ring + out * rs, capR, cap, nullptr, lane, wait, publish);
    }
    __syncthreads();
}

constexpr int MM_NWP = 8;  // warps per partition in the CTA split kernel
// resident CTAs per SM the CTA split kernel is compiled for (2: 128 registers)
#ifndef SWB_MM_MINB
#define SWB_MM_MINB 2
#endif

// Two CTAs of MM_NWP warps per (large) partition: CTA 2p runs the forward
// pass from C_s, CTA 2p + 1 the reverse pass from C_e (independent, each with
// its own ring), and the one that finishes second finds the junction on the
// middle line.  Same orientation, passes and junction rule as
// sw_mm_split_kernel.
__global__ void __launch_bounds__(32 * MM_NWP, SWB_MM_MINB) sw_mm_split_cta_kernel(const __grid_constant__ MMArgs g)
{
    __shared__ int s_gen[MM_NWP + 1], s_cols[MM_NWP + 1];
    __shared__ unsigned long long s_key;
    __shared__ int s_last;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int p = blockIdx.x >> 1, pass = blockIdx.x & 1;
    if (p >= g.nparts) return;
    const MMPart Pt = g.parts[p];
    const bool tr = (Pt.j_e - Pt.j_s) > (Pt.i_e - Pt.i_s);
    const unsigned char *X = tr ? g.B : g.A, *Y = tr ? g.A : g.B;
    const int xs = tr ? Pt.j_s : Pt.i_s, xe = tr ? Pt.j_e : Pt.i_e;
    const int ys = tr ? Pt.i_s : Pt.j_s, ye = tr ? Pt.i_e : Pt.j_e;
    auto sw12 = [&](int t) { return tr ? (t == 1 ? 2 : t == 2 ? 1 : 0) : t; };
    const int ts = sw12(Pt.t_s), te = sw12(Pt.t_e);
    const int H = xe - xs, Wd = ye - ys, mid = H / 2;
    const long long rsz = Wd + 1;
    int2 *capf = g.scratch + Pt.off;
    int2 *capr = capf + rsz;
    int2 *ring = capr + rsz + pass * (MM_NWP + 1) * rsz;
    if (pass == 0) {
        DpProb F{X + xs - 1, Y + ys - 1, 1, 1, mid, Wd, ts};
        mm_cta_pass<MM_NWP>(g, F, ring, rsz, mid, capf, s_gen, s_cols, warp, lane);
    } else {
        DpProb R{X + xe, Y + ye, -1, -1, H - mid, Wd, te == 2 ? 3 : te == 1 ? 4 : 0};
        mm_cta_pass<MM_NWP>(g, R, ring, rsz, H - mid, capr, s_gen, s_cols, warp, lane);
    }
    // the last of the two passes finds the junction (threadfence-reduction order:
    // this CTA's line is written and fenced before the counter)
    if (threadIdx.x == 0) {
        __threadfence();
        s_last = atomicAdd(g.cnt + p, 1) == 1;
        s_key = 0ull;
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    long long key = -1;
    for (int b = threadIdx.x; b <= Wd; b += blockDim.x) {
        const int2 f = __ldcg(capf + b), r = __ldcg(capr + Wd - b);
        if (f.x > NEG / 2 && r.x > NEG / 2 && f.x + r.x == Pt.score) key = max(key, 2ll * b + 1);
        else if (f.y > NEG / 2 && r.y > NEG / 2 && f.y + r.y + g.go == Pt.score) key = max(key, 2ll * b);
    }
    for (int o = 16; o > 0; o >>= 1) key = max(key, __shfl_xor_sync(0xffffffffu, key, o));
    if (lane == 0 && key >= 0) atomicMax(&s_key, (unsigned long long)(key + 1));
    __syncthreads();
    if (threadIdx.x == 0) {
        MMRes out{0, 0, -1, 0};
        const long long k2 = (long long)s_key - 1;
        if (k2 >= 0) {
            const int b = (int)(k2 >> 1);
            const bool hj = k2 & 1;
            const int2 f = __ldcg(capf + b);
            const int x = xs + mid, y = ys + b;
            out.i = tr ? y : x;
            out.j = tr ? x : y;
            out.type = hj ? 0 : (tr ? 1 : 2);
            out.sub = hj ? f.x : f.y;
        }
        g.res[p] = out;
    }
}

// One warp per partition: split it at the middle of its larger dimension.
__global__ void __launch_bounds__(256) sw_mm_split_kernel(const __grid_constant__ MMArgs g)
{
    const int lane = threadIdx.x & 31;
    const int p = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (p >= g.nparts) return;
    const MMPart Pt = g.parts[p];
    const bool tr = (Pt.j_e - Pt.j_s) > (Pt.i_e - Pt.i_s);  // columns are the larger dimension: transpose
    // orientation: rows X (length H), columns Y (length Wd); types swap 1 <-> 2 when transposed
    const unsigned char *X = tr ? g.B : g.A, *Y = tr ? g.A : g.B;
    const int xs = tr ? Pt.j_s : Pt.i_s, xe = tr ? Pt.j_e : Pt.i_e;
    const int ys = tr ? Pt.i_s : Pt.j_s, ye = tr ? Pt.i_e : Pt.j_e;
    auto sw12 = [&](int t) { return tr ? (t == 1 ? 2 : t == 2 ? 1 : 0) : t; };
    const int ts = sw12(Pt.t_s), te = sw12(Pt.t_e);
    const int H = xe - xs, Wd = ye - ys, mid = H / 2;
    int2 *rowbuf = g.scratch + Pt.off;
    int2 *capf = rowbuf + (Wd + 1);
    int2 *capr = capf + (Wd + 1);
    DpProb F{X + xs - 1, Y + ys - 1, 1, 1, mid, Wd, ts};
    mm_warp_dp<0>(g, F, rowbuf, mid, capf, nullptr, lane);
    DpProb R{X + xe, Y + ye, -1, -1, H - mid, Wd, te == 2 ? 3 : te == 1 ? 4 : 0};
    mm_warp_dp<0>(g, R, rowbuf, H - mid, capr, nullptr, lane);
    __threadfence_block();
    __syncwarp();
    // junction on line `mid`: the largest column b, an H junction before an F junction
    long long key = -1;
    for (int b = lane; b <= Wd; b += 32) {
        const int2 f = capf[b], r = capr[Wd - b];
        if (f.x > NEG / 2 && r.x > NEG / 2 && f.x + r.x == Pt.score) key = max(key, 2ll * b + 1);
        else if (f.y > NEG / 2 && r.y > NEG / 2 && f.y + r.y + g.go == Pt.score) key = max(key, 2ll * b);
    }
    for (int o = 16; o > 0; o >>= 1) key = max(key, __shfl_xor_sync(0xffffffffu, key, o));
    if (lane == 0) {
        MMRes out{0, 0, -1, 0};
        if (key >= 0) {
            const int b = (int)(key >> 1);
            const bool hj = key & 1;
            const int2 f = capf[b];
            const int x = xs + mid, y = ys + b;
            out.i = tr ? y : x;
            out.j = tr ? x : y;
            out.type = hj ? 0 : (tr ? 1 : 2);  // a gap crossing the line: vertical in this orientation
            out.sub = hj ? f.x : f.y;
        }
        g.res[p] = out;
    }
}

// Stage 5: one warp per (small) partition -- full DP with traceback codes, then
// lane 0 walks from C_e back to C_s and writes the moves ('M', 'I' = gap in S0,
// 'D' = gap in S1) right-aligned in the partition's slice of h + w bytes.
__global__ void __launch_bounds__(256) sw_mm_tb_kernel(const __grid_constant__ MMArgs g)
{
    const int lane = threadIdx.x & 31;
    const int p = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (p >= g.nparts) return;
    const MMPart Pt = g.parts[p];
    const int h = Pt.i_e - Pt.i_s, w = Pt.j_e - Pt.j_s;
    const int HW = (h + 7) / 8;
    unsigned int *codes = g.codes + Pt.off_c;
    int2 *rowbuf = g.scratch + Pt.off;
    DpProb D{g.A + Pt.i_s - 1, g.B + Pt.j_s - 1, 1, 1, h, w, Pt.t_s};
    mm_warp_dp<1>(g, D, rowbuf, 0, nullptr, codes, lane);
    __threadfence_block();
    __syncwarp();
    if (lane != 0) return;
    char *out = g.moves + Pt.off_m;
    int a = h, b = w, n = 0;
    int st = Pt.t_e;  // 0 H, 1 E, 2 F
    while (a > 0 || b > 0) {
        char c;
        if (a == 0) { c = 'I'; b--; }
        else if (b == 0) { c = 'D'; a--; }
        else {
            const unsigned int code = (codes[(long long)b * HW + (a - 1) / 8] >> (4 * ((a - 1) % 8))) & 15u;
            if (st == 0) {
                const unsigned int src = code & 3u;
                if (src == 0) { c = 'M'; a--; b--; }
                else { st = src == 1 ? 2 : 1; continue; }
            } else if (st == 2) {
                c = 'D';
                st = (code & 8u) ? 2 : 0;
                a--;
            } else {
                c = 'I';
                st = (code & 4u) ? 1 : 0;
                b--;
            }
        }
        out[h + w - 1 - n] = c;
        n++;
    }
    g.nmoves[p] = n;
}

}  // namespace swb
