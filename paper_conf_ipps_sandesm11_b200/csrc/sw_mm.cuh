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
#include "sw_fill.cuh"

namespace swb {

constexpr int MM_ALPHA = 8;
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
    int nparts;
    const MMPart *parts;
    int2 *scratch;
    MMRes *res;
    unsigned int *codes;
    char *moves;
    int *nmoves;
    int *err;            // set to 2 when a spin-wait times out (watchdog)
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

// MODE 0: run rows 1..capR and store H, F of row capR (columns 0..w) in cap.
// MODE 1: run all rows and store the 4-bit traceback code of every cell:
//   bits 0-1 H source (0 diagonal, 1 F, 2 E; ties prefer that order),
//   bit 2 E extends (E(a,b-1) - G_ext >= H(a,b-1) - G_first), bit 3 F extends.
//   Layout: codes[b * HW + (a - 1) / 8], nibble (a - 1) % 8, HW = ceil(h / 8).
template <int MODE>
__device__ void mm_warp_dp(const MMArgs &g, const DpProb &P, int2 *rowbuf, int capR, int2 *cap, unsigned int *codes,
                           int lane)
{
    const int h = P.h, w = P.w, kind = P.kind;
    const int rows = MODE == 0 ? capR : h;
    const int HW = (h + 7) / 8;
    for (int b = lane; b <= w; b += 32) {
        const int2 v = make_int2(b == 0 ? 0 : mm_row0(g, kind, b), (b == 0 && kind == 2) ? 0 : NEG);
        rowbuf[b] = v;
        if (MODE == 0 && capR == 0) cap[b] = v;
    }
    if (MODE == 0 && capR > 0 && lane == 0) cap[0] = make_int2(mm_col0(g, kind, capR), mm_col0(g, kind, capR));
    __threadfence_block();
    __syncwarp();
    const int diag00 = (kind == 3 || kind == 4) ? NEG : 0;
    for (int a0 = 0; a0 < rows; a0 += MM_CHUNK) {
        const int r0 = a0 + lane * MM_ALPHA;  // this lane: rows r0 + 1 .. r0 + MM_ALPHA
        int rc[MM_ALPHA], Hp[MM_ALPHA], Ep[MM_ALPHA];
#pragma unroll
        for (int r = 0; r < MM_ALPHA; r++) {
            const int a = r0 + r + 1;
            rc[r] = a <= h ? mm_up(P.rs[(long long)a * P.rstep]) : 0x100;  // pad rows never match
            Hp[r] = mm_col0(g, kind, a);
            Ep[r] = NEG;
        }
        int hdiag = r0 == 0 ? diag00 : mm_col0(g, kind, r0);  // H(r0, b - 1) for the next column
        int hu = 0, fu = 0;
        int2 cur = (1 + lane <= w) ? rowbuf[1 + lane] : make_int2(NEG, NEG);
        int2 nxt = (33 + lane <= w) ? rowbuf[33 + lane] : make_int2(NEG, NEG);
        const int nsteps = w + 31;
        for (int k = 0; k < nsteps; k++) {
            if (k > 0 && (k & 31) == 0) {
                cur = nxt;
                const int c = k + 33 + lane;
                nxt = c <= w ? rowbuf[c] : make_int2(NEG, NEG);
            }
            int upH = __shfl_up_sync(0xffffffffu, hu, 1);
            int upF = __shfl_up_sync(0xffffffffu, fu, 1);
            const int rH = __shfl_sync(0xffffffffu, cur.x, k & 31);
            const int rF = __shfl_sync(0xffffffffu, cur.y, k & 31);
            if (lane == 0) { upH = rH; upF = rF; }
            const int b = k - lane + 1;
            if (b >= 1 && b <= w) {
                const int cc = mm_up(P.cs[(long long)b * P.cstep]);
                int hd = hdiag;
                hdiag = upH;
                unsigned int code = 0;
                int capH = 0, capF = 0;
#pragma unroll
                for (int r = 0; r < MM_ALPHA; r++) {
                    const int e = max(Ep[r] - g.ge, Hp[r] - g.gf);                // Eq. 2
                    const int f = max(upF - g.ge, upH - g.gf);                    // Eq. 3
                    const int d = hd + (rc[r] == cc ? g.ma : g.mi);               // Eq. 1 (no 0 term)
                    const int hv = max(max(e, f), d);
                    if (MODE == 1) {
                        const unsigned int src = (d >= e && d >= f) ? 0u : (f >= e ? 1u : 2u);
                        const unsigned int ext = (Ep[r] - g.ge >= Hp[r] - g.gf ? 4u : 0u) |
                                                 (upF - g.ge >= upH - g.gf ? 8u : 0u);
                        code |= (src | ext) << (4 * r);
                    }
                    if (MODE == 0 && r0 + r + 1 == capR) { capH = hv; capF = f; }
                    hd = Hp[r];
                    Hp[r] = max(hv, NEG);
                    Ep[r] = max(e, NEG);
                    upH = Hp[r];
                    upF = max(f, NEG);
                }
                hu = upH;
                fu = upF;
                if (MODE == 1 && r0 < h) codes[(long long)b * HW + r0 / 8] = code;
                if (MODE == 0 && capR > r0 && capR <= r0 + MM_ALPHA) cap[b] = make_int2(capH, capF);
                if (lane == 31) rowbuf[b] = make_int2(hu, fu);
            }
        }
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
// reader (the next warp) is done with it.  Same arithmetic as mm_warp_dp.
template <int NWP>
__device__ void mm_cta_pass(const MMArgs &g, const DpProb &P, int2 *ring, long long rs, int capR, int2 *cap,
                            volatile int *s_gen, volatile int *s_cols, int warp, int lane)
{
    constexpr int R = NWP + 1;
    const int h = P.h, w = P.w, kind = P.kind;
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
    const int diag00 = (kind == 3 || kind == 4) ? NEG : 0;
    const int nchunks = (capR + MM_CHUNK - 1) / MM_CHUNK;
    for (int c = warp; c < nchunks; c += NWP) {
        const int a0 = c * MM_CHUNK;
        const int in = c % R, out = (c + 1) % R;
        const int2 *rin = ring + in * rs;
        int2 *rout = ring + out * rs;
        if (lane == 0) {
            s_cols[out] = 0;
            __threadfence_block();
            s_gen[out] = c;
        }
        __syncwarp();
        auto wait_cols = [&](int need) {
            need = min(need, w);
            if (lane == 0 && (s_gen[in] != c - 1 || s_cols[in] < need)) {
                const unsigned long long t0 = gtimer();
                while (s_gen[in] != c - 1 || s_cols[in] < need) {
                    __nanosleep(32);
                    if (gtimer() - t0 > (unsigned long long)g.timeout_ns) { atomicExch(g.err, 2); break; }
                }
            }
            __syncwarp();
            __threadfence_block();
        };
        const int r0 = a0 + lane * MM_ALPHA;
        int rc[MM_ALPHA], Hp[MM_ALPHA], Ep[MM_ALPHA];
#pragma unroll
        for (int r = 0; r < MM_ALPHA; r++) {
            const int a = r0 + r + 1;
            rc[r] = a <= h ? mm_up(P.rs[(long long)a * P.rstep]) : 0x100;
            Hp[r] = mm_col0(g, kind, a);
            Ep[r] = NEG;
        }
        int hdiag = r0 == 0 ? diag00 : mm_col0(g, kind, r0);
        int hu = 0, fu = 0;
        wait_cols(64);
        int2 cur = (1 + lane <= w) ? __ldcg(rin + 1 + lane) : make_int2(NEG, NEG);
        int2 nxt = (33 + lane <= w) ? __ldcg(rin + 33 + lane) : make_int2(NEG, NEG);
        int capH = 0, capF = 0;
        const int nsteps = w + 31;
        for (int k = 0; k < nsteps; k++) {
            if (k > 0 && (k & 31) == 0) {
                cur = nxt;
                wait_cols(k + 64);
                const int cc2 = k + 33 + lane;
                nxt = cc2 <= w ? __ldcg(rin + cc2) : make_int2(NEG, NEG);
            }
            int upH = __shfl_up_sync(0xffffffffu, hu, 1);
            int upF = __shfl_up_sync(0xffffffffu, fu, 1);
            const int rH = __shfl_sync(0xffffffffu, cur.x, k & 31);
            const int rF = __shfl_sync(0xffffffffu, cur.y, k & 31);
            if (lane == 0) { upH = rH; upF = rF; }
            const int b = k - lane + 1;
            if (b >= 1 && b <= w) {
                const int cc = mm_up(P.cs[(long long)b * P.cstep]);
                int hd = hdiag;
                hdiag = upH;
#pragma unroll
                for (int r = 0; r < MM_ALPHA; r++) {
                    const int e = max(Ep[r] - g.ge, Hp[r] - g.gf);   // Eq. 2
                    const int f = max(upF - g.ge, upH - g.gf);       // Eq. 3
                    const int d = hd + (rc[r] == cc ? g.ma : g.mi);  // Eq. 1 (no 0 term)
                    const int hv = max(max(e, f), d);
                    if (r0 + r + 1 == capR) { capH = hv; capF = f; }
                    hd = Hp[r];
                    Hp[r] = max(hv, NEG);
                    Ep[r] = max(e, NEG);
                    upH = Hp[r];
                    upF = max(f, NEG);
                }
                hu = upH;
                fu = upF;
                if (capR > r0 && capR <= r0 + MM_ALPHA) cap[b] = make_int2(capH, capF);
                if (lane == 31) rout[b] = make_int2(hu, fu);
            }
            if ((k & 31) == 31 || k == nsteps - 1) {
                __threadfence_block();
                __syncwarp();
                if (lane == 31) s_cols[out] = min(w, k - 30);
            }
        }
    }
    __syncthreads();
}

constexpr int MM_NWP = 8;  // warps per partition in the CTA split kernel

// One CTA of MM_NWP warps per (large) partition: split it at the middle of
// its larger dimension.  Same orientation, passes and junction rule as
// sw_mm_split_kernel.
__global__ void __launch_bounds__(32 * MM_NWP) sw_mm_split_cta_kernel(const __grid_constant__ MMArgs g)
{
    __shared__ int s_gen[MM_NWP + 1], s_cols[MM_NWP + 1];
    __shared__ unsigned long long s_key;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int p = blockIdx.x;
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
    int2 *ring = g.scratch + Pt.off;
    int2 *capf = ring + (MM_NWP + 1) * rsz;
    int2 *capr = capf + rsz;
    DpProb F{X + xs - 1, Y + ys - 1, 1, 1, mid, Wd, ts};
    mm_cta_pass<MM_NWP>(g, F, ring, rsz, mid, capf, s_gen, s_cols, warp, lane);
    DpProb R{X + xe, Y + ye, -1, -1, H - mid, Wd, te == 2 ? 3 : te == 1 ? 4 : 0};
    mm_cta_pass<MM_NWP>(g, R, ring, rsz, H - mid, capr, s_gen, s_cols, warp, lane);
    if (threadIdx.x == 0) s_key = 0ull;
    __syncthreads();
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
