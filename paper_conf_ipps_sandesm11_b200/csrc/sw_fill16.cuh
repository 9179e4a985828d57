// sw_fill16.cuh -- packed 16x2 Stage-1 fill.
//
// Same band pipeline, I/O warp, row border, special rows, stripes and exact
// best-cell replay as sw_fill.cuh (read that first); what changes is the lane:
//
//  * A lane owns 2 NS rows (NS = 8, 15 or 16) as NS packed slots: slot s holds
//    row s in its low half at column j and row s+NS in its high half at
//    column j-1, so ONE instruction updates two cells that do not depend on
//    each other.  Slot 0's high half takes row NS-1's values of the previous
//    step (a PRMT), so the vertical chain is NS slots long instead of 2 NS.
//  * Values are biased unsigned 16-bit numbers in a warp-uniform frame
//    q = x - B + 32768 (x the int32 value), re-based at every tile.  Within a
//    warp all live values lie within ~650 (p_max + G_first) of each other
//    (|H(i,j) - H(i-1,j)| <= p_max + G_first), far inside
//    16 bits for the supported scorings, so the frame never wraps.
//  * Adds that cannot borrow across halves are plain 32-bit adds on the FMA
//    pipe (q - G_ext, q - G_first); the signed substitution score is added
//    with the per-half VIADDMNMX.U16x2; t and the next row's F are one
//    VIADDMNMX.U16x2 each from (F, D - G_first) (cell_hf, SWB_FMODE 2); maxima
//    use VIMNMX3.U16x2.  The local 0 floor is the frame's image of 0; the
//    global (reverse-pass) instantiation has no floor.
//  * The gap penalties are compile-time magic immediates in the patchable
//    build (SWB_PATCH, sw_fill16_patch.cu) that the library rewrites per
//    scoring: an add with an immediate reads one register instead of three.
//  * Everything that leaves the lane (warp ring, special rows, the right
//    border of a stripe, replay tracking) is converted back to int32.
//
// Results are bit-identical to the int32 kernel at every real cell; the two
// differences are internal and exact: E(i,0) and F(0,j) start at t instead of
// -infinity (both give E(i,1) = t(i,0), F(1,j) = t(0,j)), and pad columns use
// base code 0 (they only feed pad cells; tracking ignores them).
#pragma once
#include "sw_fill.cuh"

namespace swb {

constexpr int BIAS16 = 32768;
#ifndef SWB_FMODE
#define SWB_FMODE 2
#endif
// Magic immediates of the patchable build (sw_fill16_patch.cu): -G_ext and
// -G_first in both halves as a 32-bit add (NGE2, NGF2) and per half (NGE16,
// NGF16).  Arbitrary values, chosen not to occur elsewhere in the code.
#ifndef SWB_K_NGE2
#define SWB_K_NGE2 0x6b8b4567u
#define SWB_K_NGF2 0x327b23c6u
#define SWB_K_NGE16 0x643c9869u
#define SWB_K_NGF16 0x66334873u
#endif
#ifndef SWB_ADDMODE
#define SWB_ADDMODE 1  // plain adds; 0: IMAD with a runtime 1
#endif
// Lane steps per iteration of the fast tile loop: 8 for the local-mode
// geometries with 8 or more warps or 15 slots, 4 otherwise (4 warps x 16
// slots: 9.2 -> 14.0 ms on C1 at 8; measured); SWB_UNR
// overrides it for every geometry.
#ifndef SWB_UNR
#define SWB_UNR 0
#endif
// Lane steps per iteration in the special-row tiles (SPM 1 / 2 / 3); 0: as SWB_UNR's
// rule.  4: the warp with a special row runs a different loop than its CTA's other
// warps; a shorter body keeps both hot loops in the instruction cache (C4, alpha 34,
// k = 131072: 21.4 -> 19.9 s; profiles/r02_spm3.txt).
#ifndef SWB_SPU
#define SWB_SPU 4
#endif


__device__ __forceinline__ uint32_t pk(int lo, int hi) { return (uint32_t)(lo & 0xffff) | ((uint32_t)hi << 16); }
__device__ __forceinline__ int lo16(uint32_t v) { return (int)(v & 0xffffu); }
__device__ __forceinline__ int hi16(uint32_t v) { return (int)(v >> 16); }

// Per-column selector parts for the packed PRMT: low byte = nibbles selecting
// P[c] with sign replication (low half), high byte = nibbles selecting Q[c]
// (bytes 4..7) for the high half.
__device__ __forceinline__ uint32_t col_sel16(uint32_t code)
{
    const uint32_t lo = code | ((code | 8u) << 4);
    const uint32_t hi = (code + 4u) | (((code + 4u) | 8u) << 4);
    return lo | (hi << 8);
}

template <int NW, int W, int NS = 8, bool SPLIT = false, bool LOCAL = true>
struct Fill16 {
    static constexpr int ALPHA = 2 * NS, BH = ALPHA * 32 * NW;
    static constexpr int RING = Smem<W, NW>::RING;
    static constexpr int SRING = Smem<W, NW>::SRING;
    static constexpr int SKEW = 63;     // lane 31's output column lags lane 0's by 2*31 + 1
    static constexpr int STEPS = W;     // one column per lane step
    static constexpr int UNR = SWB_UNR > 0 ? SWB_UNR : (LOCAL && (NW >= 8 || NS == 15)) ? 8 : 4;
    static constexpr int NSAVE = 2 * NS + 3;
    static constexpr int SPB = 128;  // SPM 3 staging entries per warp (two tiles of columns)
    static constexpr int HALF = SRING / 2 + 32;  // selector ring: one parity half + a 32-entry mirror
    // Warp-to-warp rings of (t, F): column col lives at ridx(col) in [1, RING]
    // (stride RS = RING + 1), so the 64 columns k0 - 63 .. k0 a lane-31 tile
    // writes (k0 a multiple of 64) sit at consecutive indices from
    // ((k0 - 64) & (RING - 1)) + 1: immediate offsets, no wrap.
    static constexpr int RS = RING + 1;
    static __device__ __forceinline__ int ridx(int col) { return ((col - 1) & (RING - 1)) + 1; }
    static_assert(W % 64 == 0 && W > SKEW, "W multiple of 64, larger than the warp skew");
    static_assert(W == 64, "the converted-ring and selector addressing assume 64-column tiles");

    // rings (int2, (NW+1) x RS) | selectors (2 x HALF u32) | converted ring (NW x W u32) | saves
    static size_t smem_bytes()
    {
        return sizeof(int2) * RS * (NW + 1) + sizeof(uint32_t) * 2 * HALF + sizeof(uint32_t) * NW * W +
               sizeof(int) * NSAVE * 32 * NW + sizeof(uint2) * SPB * NW;
    }

    struct Lane {
        uint32_t P[NS], Q[NS];  // int8x4 profiles of rows s (low halves) and s+NS (high halves)
        uint32_t e[NS], t[NS];  // packed E and t = H - G_first of the previous column of each half
        uint32_t tprev;       // packed diagonal input of slot 0
        uint32_t fn;          // packed F of the rows after the last slot (low: row NS at j, high: row 2NS at j-1)
        int B;                // warp-uniform frame base
        int adj;              // BIAS16 - B: int32 value -> frame
        int Bm;               // B - BIAS16: frame -> int32 value
        uint32_t FL;          // packed frame image of the local floor 0
    };

    // Selector ring layout: even columns in the first half, odd in the second,
    // so the 32 lanes of a step (columns k - 2 lane, all of one parity) read
    // 32 consecutive words: no bank conflicts.  Each half has a 32-word mirror
    // of its first 32 words, so a lane's 64 steps of a tile read
    // base + (kk >> 1) + (kk & 1) * HALF without wrapping (immediate offsets).
    // The word of column c is the complete PRMT selector of a lane step whose
    // low half is at c and high half at c - 1.
    static __device__ __forceinline__ void put_sel(uint32_t *selr, int col, uint32_t code, uint32_t code_left)
    {
        const uint32_t c = (uint32_t)col & (SRING - 1), h = c >> 1, par = c & 1u;
        const uint32_t v = (col_sel16(code) & 0xffu) | (col_sel16(code_left) & 0xff00u);
        selr[par * HALF + h] = v;
        if (h < 32) selr[par * HALF + h + SRING / 2] = v;
    }

    static __device__ __forceinline__ int toabs(const Lane &L, int q) { return q + L.Bm; }
    static __device__ __forceinline__ int tofr(const Lane &L, int x) { return x - L.B + BIAS16; }

    // One lane step: low half at local column jl = k - 2 lane, high half at jl - 1.
    //
    // Cell update, with D = max(H_diag + p, E, 0) (so H = max(D, F), Eq. 1):
    //   E*  = max(E*_left - G_ext, t_left, 0)     Eq. 2, floored at 0 (below)
    //   D   = max(t_diag + (p + G_first), E*)
    //   H   = max(D, F);  t = H - G_first
    //   F'  = max(F - G_ext, D - G_first)         Eq. 3 for the next row
    // F' = max(F - G_ext, t) = max(F - G_ext, D - G_first, F - G_first) and
    // G_ext <= G_first, so the F chain down the lane's rows is one max per row
    // and D (which only needs the previous column) is off that chain.
    // Flooring E at 0 is exact for H and F: max(E, 0) satisfies the same
    // recurrence (max(max(E,0) - G_ext, t, 0) = max(E - G_ext, t, 0)), and H
    // takes max(.., E, .., 0) anyway.  E only leaves the lane as a stripe's
    // right border, where the receiver's H and F are unchanged by the floor.
    // H, t and the next row's F of one slot from D and the incoming F (both
    // halves).  SWB_FMODE selects the instruction mix:
    //   0: H = max(D, F); t = H - G_first; F' = max(F - G_ext, D - G_first)
    //      (IMAD + VIMNMX on the F chain)
    //   1: F' = VIADDMNMX(F, -G_ext, D - G_first): the F chain down the slots
    //      is one same-pipe instruction per slot
    //   2: as 1, and t = VIADDMNMX(F, -G_first, D - G_first) directly; the
    //      tile maximum is then taken over t (= H - G_first) instead of H,
    //      except in replays (TRACK), which need H.
    // The u16x2 adds never wrap: every frame value stays far above G_first.
    // x + c (both halves; never borrows, see above).  SWB_ADDMODE 1 (default):
    // a plain add -- an immediate-form VIADD (FMA pipe, one register read) in
    // the patched image, IMAD R, R, imm, R (two reads) otherwise; 0: IMAD with
    // a runtime 1 (three reads, measured 4-10 % slower).
    static __device__ __forceinline__ uint32_t add_fma(uint32_t x, int one, int c)
    {
        if constexpr (SWB_ADDMODE == 0) return (uint32_t)imad((int)x, one, c);
        else return x + (uint32_t)c;
    }

    template <bool TRACK>
    static __device__ __forceinline__ void cell_hf(uint32_t d, uint32_t &fu, uint32_t &h, uint32_t &t, int one,
                                                   int nge2, int ngf2, uint32_t nge16, uint32_t ngf16)
    {
        if constexpr (SWB_FMODE == 0) {
            h = __vmaxu2(d, fu);
            t = (uint32_t)imad((int)h, one, ngf2);
            fu = __vmaxu2((uint32_t)imad((int)fu, one, nge2), (uint32_t)imad((int)d, one, ngf2));
        } else {
            const uint32_t dg = add_fma(d, one, ngf2);
            if constexpr (SWB_FMODE == 1 || TRACK) {
                h = __vmaxu2(d, fu);
                t = (uint32_t)imad((int)h, one, ngf2);
            } else if constexpr (SWB_FMODE >= 3) {
                // t = max(F - G_first, D - G_first) as an FMA-pipe add and a
                // full-rate max (one ALU cycle instead of two)
                t = __vmaxu2(add_fma(fu, one, ngf2), dg);
                h = t;
            } else {
                t = __viaddmax_u16x2(fu, ngf16, dg);
                h = t;
            }
            if constexpr (SWB_FMODE == 4 && !TRACK) fu = __vmaxu2(add_fma(fu, one, nge2), dg);
            else fu = __viaddmax_u16x2(fu, nge16, dg);
        }
    }
    // Offset from the tile maximum a non-replay tile returns to H (mode 2: t).
    static __device__ __forceinline__ int tmax_off(const FillArgs &a) { return SWB_FMODE >= 2 && !SPLIT ? a.gf : 0; }

    // SPM: 0 no special row in the warp; 1 special rows are strip bottoms (the
    // high half of the last slot); 2 one special row per lane anywhere in the
    // strip (k >= alpha, host rule): strip row sp_r (< NS: slot sp_r's low half,
    // else slot sp_r - NS's high half, one column behind), -1 none -- a tail
    // segment whose first row is not a multiple of alpha, or k not a multiple of
    // alpha.  The slot loop only selects that slot's (t, F) (two SELs per slot);
    // one store pair after the loop.
    // SPM 3: as SPM 2 for a warp with exactly one such lane (X.splane, k >= 32
    // alpha): that lane stages the packed (t, F) pair in shared memory (X.spb,
    // one STS per step) and the warp writes the tile's columns coalesced after
    // the tile (sw_fill16_kernel sp_flush) instead of two guarded global stores
    // per step.  SPS >= 0 (SPM 2 / 3): the special row's slot is SPS in every
    // lane that has one (warp-uniform, known at compile time), so the capture is
    // two register moves at that slot instead of a compare and two selects per slot.
    template <bool GUARD, bool TRACK, int SPM, bool CAP, int SPS = -1>
    static __device__ __forceinline__ uint32_t step(const FillArgs &a, const StepInfo &X, Lane &L, int k, int lane,
                                                    uint32_t cr_a, uint32_t ro_a, uint32_t sel_a, uint32_t pt_sel,
                                                    int one, uint32_t tmax, int row1, int &bs, int &bi, int &bj,
                                                    int *sp_ptr, int sp_r)
    {
        const int sp_s = SPS >= 0 ? SPS : sp_r < NS ? sp_r : sp_r - NS;  // the slot of the lane's special row (SPM 2)
        uint32_t sp_t = 0u, sp_f = 0u;
        const uint32_t up_t = __shfl_up_sync(0xffffffffu, L.t[NS - 1], 1);
        const uint32_t up_f = __shfl_up_sync(0xffffffffu, L.fn, 1);
        const int jl = k - 2 * lane;
        // lane 0: the warp above's bottom row at column jl, already in this warp's
        // frame (converted at tile start): low half t, high half F of row 0.
        uint32_t cr, sel;
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(cr) : "r"(cr_a) : "memory");
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(sel) : "r"(sel_a) : "memory");
        Lane S;
        if (GUARD) S = L;
        if (TRACK) tmax = 0;
        const uint32_t tmax_in = tmax;
        // slot-0 inputs: low = upper lane's row 15 (its high half) or the ring, high = own row 7
        uint32_t tu = __byte_perm(lane == 0 ? cr : up_t, L.t[NS - 1], pt_sel);
        uint32_t fu = __byte_perm(lane == 0 ? cr : up_f, L.fn, 0x5432);  // F of slot 0's rows
        uint32_t td = L.tprev;
        L.tprev = tu;
#if defined(SWB_PATCH)
        // Instruction immediates that sw_api.cu patches in the cubin at load
        // time with this call's values: an add with an
        // immediate reads one register instead of three.
        constexpr int nge2 = (int)SWB_K_NGE2, ngf2 = (int)SWB_K_NGF2;
        constexpr uint32_t nge16 = SWB_K_NGE16, ngf16 = SWB_K_NGF16;
#else
        const int nge2 = -(a.ge * 0x10001), ngf2 = -(a.gf * 0x10001);
        // per-half two's complements of -G_ext, -G_first for the u16x2 adds
        const uint32_t nge16 = ((0x10000u - (uint32_t)a.ge) & 0xffffu) * 0x10001u;
        const uint32_t ngf16 = ((0x10000u - (uint32_t)a.gf) & 0xffffu) * 0x10001u;
#endif
        uint32_t f15 = 0;  // F entering the last slot (row 2NS-1 in the high half)
        if constexpr (SPLIT) {
            // Same cells, shorter F chain for latency-bound warps: D of every slot
            // first (it only needs the previous column), then F down the rows as two
            // half chains.  The second starts from D - G_first of the slot before
            // it, a lower bound of the true F there, and is corrected by
            // F_s = max(partial_s, F_h - (s - h) G_ext), h = NS/2 (the F recurrence
            // is a max-plus scan: F_s = max over s' < s of (D_s' - G_first - (s-s'-1) G_ext)
            // together with F_0 - s G_ext).
            uint32_t d[NS];
#pragma unroll
            for (int s = 0; s < NS; s++) {
                const uint32_t e0 = __vimax3_u16x2(add_fma(L.e[s], one, nge2), L.t[s], L.FL);
                const uint32_t p0 = (uint32_t)prmt(L.P[s], L.Q[s], sel);
                d[s] = __viaddmax_u16x2(td, p0, e0);
                td = L.t[s];
                L.e[s] = e0;
                if (CAP) {
                    if (jl == X.jcap) X.rbrow[s].y = toabs(L, lo16(e0));
                    if (jl - 1 == X.jcap) X.rbrow[s + NS].y = toabs(L, hi16(e0));
                }
            }
            constexpr int HS = NS / 2;
            uint32_t fa = fu, fb = (uint32_t)imad((int)d[HS - 1], one, ngf2);
            uint32_t F[NS];
#pragma unroll
            for (int s = 0; s < HS; s++) {
                F[s] = fa;
                fa = __vmaxu2((uint32_t)imad((int)fa, one, nge2), (uint32_t)imad((int)d[s], one, ngf2));
                F[HS + s] = fb;
                fb = __vmaxu2((uint32_t)imad((int)fb, one, nge2), (uint32_t)imad((int)d[HS + s], one, ngf2));
            }
            // fa = F_HS; correct the second half and the outgoing F
#pragma unroll
            for (int s = 1; s < HS; s++) F[HS + s] = __vmaxu2(F[HS + s], (uint32_t)imad((int)fa, one, -(s * a.ge * 0x10001)));
            F[HS] = fa;
            fu = __vmaxu2(fb, (uint32_t)imad((int)fa, one, -(HS * a.ge * 0x10001)));
            f15 = F[NS - 1];
#pragma unroll
            for (int s = 0; s < NS; s += 2) {
                const uint32_t h0 = __vmaxu2(d[s], F[s]), h1 = __vmaxu2(d[s + 1], F[s + 1]);
                L.t[s] = (uint32_t)imad((int)h0, one, ngf2);
                L.t[s + 1] = (uint32_t)imad((int)h1, one, ngf2);
                tmax = __vimax3_u16x2(tmax, h0, h1);
                if (CAP) {
                    if (jl == X.jcap) {
                        X.rbrow[s].x = toabs(L, lo16(L.t[s]));
                        X.rbrow[s + 1].x = toabs(L, lo16(L.t[s + 1]));
                    }
                    if (jl - 1 == X.jcap) {
                        X.rbrow[s + NS].x = toabs(L, hi16(L.t[s]));
                        X.rbrow[s + NS + 1].x = toabs(L, hi16(L.t[s + 1]));
                    }
                }
            }
        } else {
#pragma unroll
            for (int s = 0; s < NS; s += 2) {
                const uint32_t e0 = __vimax3_u16x2(add_fma(L.e[s], one, nge2), L.t[s], L.FL);
                const uint32_t p0 = (uint32_t)prmt(L.P[s], L.Q[s], sel);
                const uint32_t d0 = __viaddmax_u16x2(td, p0, e0);
                td = L.t[s];
                uint32_t h0, t0;
                if (s == NS - 1) f15 = fu;  // odd NS: the last slot is unpaired
                const uint32_t fin0 = fu;   // F of slot s's rows (SPM 2)
                cell_hf<TRACK>(d0, fu, h0, t0, one, nge2, ngf2, nge16, ngf16);
                L.e[s] = e0;
                L.t[s] = t0;
                if (SPM >= 2 && !TRACK && (SPS >= 0 ? s == SPS : s == sp_s)) { sp_t = t0; sp_f = fin0; }
                if (s + 1 == NS) {
                    tmax = __vmaxu2(tmax, h0);
                    if (CAP) {
                        if (jl == X.jcap) X.rbrow[s] = make_int2(toabs(L, lo16(t0)), toabs(L, lo16(e0)));
                        if (jl - 1 == X.jcap) X.rbrow[s + NS] = make_int2(toabs(L, hi16(t0)), toabs(L, hi16(e0)));
                    }
                    break;
                }
                if (s == NS - 2) f15 = fu;
                const uint32_t e1 = __vimax3_u16x2(add_fma(L.e[s + 1], one, nge2), L.t[s + 1], L.FL);
                const uint32_t p1 = (uint32_t)prmt(L.P[s + 1], L.Q[s + 1], sel);
                const uint32_t d1 = __viaddmax_u16x2(td, p1, e1);
                td = L.t[s + 1];
                uint32_t h1, t1;
                const uint32_t fin1 = fu;
                cell_hf<TRACK>(d1, fu, h1, t1, one, nge2, ngf2, nge16, ngf16);
                L.e[s + 1] = e1;
                L.t[s + 1] = t1;
                if (SPM >= 2 && !TRACK && (SPS >= 0 ? s + 1 == SPS : s + 1 == sp_s)) { sp_t = t1; sp_f = fin1; }
                tmax = __vimax3_u16x2(tmax, h0, h1);  // TRACK: this step's maximum (reset per step)
                if (CAP) {
                    if (jl == X.jcap) {
                        X.rbrow[s] = make_int2(toabs(L, lo16(t0)), toabs(L, lo16(e0)));
                        X.rbrow[s + 1] = make_int2(toabs(L, lo16(t1)), toabs(L, lo16(e1)));
                    }
                    if (jl - 1 == X.jcap) {
                        X.rbrow[s + NS] = make_int2(toabs(L, hi16(t0)), toabs(L, hi16(e0)));
                        X.rbrow[s + NS + 1] = make_int2(toabs(L, hi16(t1)), toabs(L, hi16(e1)));
                    }
                }
            }
        }
        L.fn = fu;
        if (GUARD) {
            // lanes left of column 0 keep their state; at jl == 0 only the high half waits
            const uint32_t keep = (jl >= 0 ? 0x0000ffffu : 0u) | (jl >= 1 ? 0xffff0000u : 0u);
#pragma unroll
            for (int s = 0; s < NS; s++) {
                L.e[s] = (L.e[s] & keep) | (S.e[s] & ~keep);
                L.t[s] = (L.t[s] & keep) | (S.t[s] & ~keep);
            }
            if (jl < 0) {
                L.tprev = S.tprev;
                L.fn = S.fn;
            }
            tmax = (tmax & keep) | (tmax_in & ~keep);
        }
        if (TRACK && !LOCAL) {
            // Replay of a reverse (global) pass: the first cell in row-major
            // order with H == goal (reading S10).  Within a step a row occurs
            // once and the low half's rows precede the high half's; across
            // steps the running (bi, bj) keeps the lexicographic minimum.
            // Columns past X.hw cannot hold a start.
            const int gq = a.goal - a.gf - L.B + BIAS16;  // goal's t in this warp's frame
            if (gq >= 0 && gq <= 0xffff) {
                const uint32_t Gt = (uint32_t)gq * 0x10001u;
                const bool lo_ok = jl >= 0 && jl < X.hw, hi_ok = jl >= 1 && jl - 1 < X.hw;
                uint32_t lob = 0u, hib = 0u;
#pragma unroll
                for (int s = 0; s < NS; s++) {
                    const uint32_t eq = __vcmpeq2(L.t[s], Gt);
                    lob |= (eq & 1u) << s;
                    hib |= (eq >> 31) << s;
                }
                lob = lo_ok ? lob : 0u;
                hib = hi_ok ? hib : 0u;
                if (lob | hib) {
                    int row, col;
                    if (lob) { row = row1 + __ffs(lob) - 1; col = X.col0 + jl + 1; }
                    else { row = row1 + NS + __ffs(hib) - 1; col = X.col0 + jl; }
                    if (row <= a.m && (row < bi || (row == bi && col < bj))) { bi = row; bj = col; }
                }
            }
            return 0;
        }
        if (TRACK) {
            // Replay: the step's cells are t[s] + G_first now.  The best cell
            // of the step (max, then min row; a row occurs once per step) is
            // the only one that can beat the running best.  Halves outside
            // the stripe's columns are masked; a pad row (> m) never holds a
            // step maximum that beats the best (its F is below an H of a real
            // row of the same column, examined at this or the previous step,
            // and rows are scanned in increasing order).
            const bool lo_ok = jl >= 0 && jl < X.w, hi_ok = jl >= 1 && jl - 1 < X.w;
            const uint32_t vm = (lo_ok ? 0x0000ffffu : 0u) | (hi_ok ? 0xffff0000u : 0u);
            const uint32_t tm = tmax & vm;
            const int M = max(lo16(tm), hi16(tm));
            if (vm != 0u && toabs(L, M) >= max(bs, 1)) {
                const uint32_t Mt = (uint32_t)(M - a.gf) * 0x10001u;
                uint32_t lob = 0u, hib = 0u;
#pragma unroll
                for (int s = 0; s < NS; s++) {
                    const uint32_t eq = __vcmpeq2(L.t[s], Mt);
                    lob |= (eq & 1u) << s;
                    hib |= (eq >> 31) << s;
                }
                lob = lo_ok ? lob : 0u;
                hib = hi_ok ? hib : 0u;
                int row, col;
                if (lob) { row = row1 + __ffs(lob) - 1; col = X.col0 + jl + 1; }
                else { row = row1 + NS + __ffs(hib) - 1; col = X.col0 + jl; }
                const int v = toabs(L, M);
                if ((lob | hib) && row <= a.m && better(v, row, col, bs, bi, bj)) { bs = v; bi = row; bj = col; }
            }
            return 0;
        }
        const int jo = jl - 1;  // row 2NS-1's column (high half of the last slot)
        if (SPM == 2 && !SPLIT && sp_ptr != nullptr) {
            const int hi = sp_r >= NS ? 1 : 0, col = jl - hi;
            if (col >= 0 && col < X.w) {
                sp_ptr[col] = toabs(L, hi ? hi16(sp_t) : lo16(sp_t)) + a.gf;  // H = t + G_first
                sp_ptr[X.sp_ld + col] = toabs(L, hi ? hi16(sp_f) : lo16(sp_f));
            }
        }
        if (SPM == 3 && lane == X.splane)
            asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(X.spb + 8u * ((uint32_t)jl & (SPB - 1))), "r"(sp_t), "r"(sp_f)
                         : "memory");
        if (SPM == 1 && sp_ptr != nullptr && jo >= 0 && jo < X.w) {
            sp_ptr[jo] = toabs(L, hi16(L.t[NS - 1])) + a.gf;  // H = t + G_first
            sp_ptr[X.sp_ld + jo] = toabs(L, hi16(f15));
        }
        if (!TRACK && lane == 31 && (!GUARD || jo >= 0)) {
            // (t, F) of row 15 at column jo for the next warp (int32, absolute)
            asm volatile("st.shared.v2.s32 [%0], {%1, %2};" ::"r"(ro_a),
                         "r"(toabs(L, hi16(L.t[NS - 1]))), "r"(toabs(L, hi16(f15))) : "memory");
        }
        return tmax;
    }

    // Lane 0's ring input of this tile, converted once into the warp's frame:
    // cring[x] = t | F' << 16 for column c*W + x, F' = max(F - G_ext, t) the F of
    // the warp's first row.  Warp w-1 finished these columns LAG tiles ago.
    static __device__ __forceinline__ void convert_ring(const FillArgs &a, const Lane &L, const int2 *ring_in,
                                                        uint32_t *cring, int c, int lane)
    {
#pragma unroll
        for (int x = lane; x < W; x += 32) {
            const int2 v = ring_in[ridx(c * W + x)];
            cring[x] = (uint32_t)((v.x + L.adj) & 0xffff) | ((uint32_t)(max(v.y - a.ge, v.x) + L.adj) << 16);
        }
        __syncwarp();
    }

    template <bool GUARD, bool TRACK, int SPM, bool CAP, int SPS = -1>
    static __device__ __forceinline__ uint32_t tile(const FillArgs &a, const StepInfo &X, Lane &L, int c, int lane,
                                                    uint32_t cring, uint32_t ring_out, uint32_t selr, int row1,
                                                    int &bs, int &bi, int &bj, int *sp_ptr, int sp_r)
    {
        uint32_t tmax = 0;
        const int k0 = c * STEPS;
        const uint32_t pt_sel = lane == 0 ? 0x5410u : 0x5432u;
        const int one = (int)pin((uint32_t)a.one);
        // this lane's selector words: column k0 + kk - 2 lane
        const uint32_t sel0 = selr + 4u * ((((uint32_t)(k0 - 2 * lane)) & (SRING - 1)) >> 1);
        // lane 31's ring output: column k0 + kk - 63 at ridx = base + kk
        const uint32_t ro0 = ring_out + 8u * (uint32_t)(((k0 - 64) & (RING - 1)) + 1);
        if (GUARD || TRACK || CAP) {
#pragma unroll 1
            for (int kk = 0; kk < STEPS; kk++)
                tmax = step<GUARD, TRACK, SPM, CAP>(a, X, L, k0 + kk, lane, cring + 4u * kk, ro0 + 8u * kk,
                                                    sel0 + 4u * ((kk >> 1) + (kk & 1) * HALF), pt_sel, one, tmax,
                                                    row1, bs, bi, bj, sp_ptr, sp_r);
        } else {
            // special-row tiles run next to the other warps' SPM-0 loop: a shorter
            // body keeps both hot loops in the instruction cache (SWB_SPU)
            constexpr int U = SPM == 0 ? UNR : (SWB_SPU > 0 ? SWB_SPU : UNR);
#pragma unroll 1
            for (int kq = 0; kq < STEPS; kq += U) {
                const uint32_t sq = sel0 + 2u * kq, cq = cring + 4u * kq, oq = ro0 + 8u * kq;
#pragma unroll
                for (int u = 0; u < U; u++)
                    tmax = step<false, false, SPM, false, SPS>(a, X, L, k0 + kq + u, lane, cq + 4u * u, oq + 8u * u,
                                                          sq + 4u * ((u >> 1) + (u & 1) * HALF), pt_sel, one, tmax,
                                                          row1, bs, bi, bj, sp_ptr, sp_r);
            }
        }
        return tmax;
    }

    // The fast SPM-3 tile with the special row's slot sps as a compile-time
    // constant: one instantiation per slot.
    template <int S = 0>
    static __device__ __forceinline__ uint32_t tile_gen(int sps, const FillArgs &a, const StepInfo &X, Lane &L, int c,
                                                        int lane, uint32_t cring, uint32_t ring_out, uint32_t selr,
                                                        int row1, int &bs, int &bi, int &bj, int *sp_ptr, int sp_r)
    {
        if constexpr (S < NS) {
            if (sps == S) return tile<false, false, 3, false, S>(a, X, L, c, lane, cring, ring_out, selr, row1, bs, bi, bj, sp_ptr, sp_r);
            return tile_gen<S + 1>(sps, a, X, L, c, lane, cring, ring_out, selr, row1, bs, bi, bj, sp_ptr, sp_r);
        } else {
            return tile<false, false, 3, false>(a, X, L, c, lane, cring, ring_out, selr, row1, bs, bi, bj, sp_ptr, sp_r);
        }
    }

    // Re-base the frame to lane 0's slot-0 low value (warp-uniform shift).
    static __device__ __forceinline__ void rebase(const FillArgs &a, Lane &L)
    {
        const int d = __shfl_sync(0xffffffffu, lo16(L.t[0]), 0) - BIAS16;
        const int d2 = -(d * 0x10001);
#pragma unroll
        for (int s = 0; s < NS; s++) {
            L.e[s] = (uint32_t)imad((int)L.e[s], a.one, d2);
            L.t[s] = (uint32_t)imad((int)L.t[s], a.one, d2);
        }
        L.tprev = (uint32_t)imad((int)L.tprev, a.one, d2);
        L.fn = (uint32_t)imad((int)L.fn, a.one, d2);
        L.B += d;
        L.adj = BIAS16 - L.B;
        L.Bm = L.B - BIAS16;
        const int fl = LOCAL ? min(max(BIAS16 - L.B, 0), 0xffff) : 0;  // global: no 0 floor
        L.FL = (uint32_t)fl * 0x10001u;
    }

    static __device__ __forceinline__ void save(const Lane &L, int *sv, int lane)
    {
#pragma unroll
        for (int s = 0; s < NS; s++) {
            sv[s * 32 + lane] = (int)L.e[s];
            sv[(NS + s) * 32 + lane] = (int)L.t[s];
        }
        sv[(2 * NS) * 32 + lane] = (int)L.tprev;
        sv[(2 * NS + 1) * 32 + lane] = (int)L.fn;
        sv[(2 * NS + 2) * 32 + lane] = L.B;
    }
    static __device__ __forceinline__ void restore(Lane &L, const int *sv, int lane)
    {
#pragma unroll
        for (int s = 0; s < NS; s++) {
            L.e[s] = (uint32_t)sv[s * 32 + lane];
            L.t[s] = (uint32_t)sv[(NS + s) * 32 + lane];
        }
        L.tprev = (uint32_t)sv[(2 * NS) * 32 + lane];
        L.fn = (uint32_t)sv[(2 * NS + 1) * 32 + lane];
        L.B = sv[(2 * NS + 2) * 32 + lane];
        L.adj = BIAS16 - L.B;
        L.Bm = L.B - BIAS16;
        const int fl = LOCAL ? min(max(BIAS16 - L.B, 0), 0xffff) : 0;
        L.FL = (uint32_t)fl * 0x10001u;
    }
};

// COOP = false: NW compute warps + one I/O warp.  COOP = true: NW compute
// warps that also share the I/O (each loads and drains W / NW columns per
// tile), so all four SMSPs carry the same number of compute warps (16 warps:
// 4 each) -- the lockstep interval otherwise waits for the busier SMSPs.
// LOCAL = false: the reverse pass of sw_reverse_goal (a8): anchored global
// recurrence with no 0 floor (FL = 0), global boundaries, first-hit tracking of
// the goal and the early exit after the band with the first hit, as in the
// int32 kernel; one stripe, no special rows, no Stage-2 matching (host checks).
// GEN = true: also the generic special-row tiles (SPM 2: a special row that is
// not a strip bottom -- k not a multiple of alpha, or a tail segment whose first
// row is not); a separate instantiation, so the strip-bottom kernels keep their
// code (the generic tiles cost the GEN kernel ~2 % on C4).
template <int NW, int W, bool COOP = false, int NS = 8, bool SPLIT = false, bool LOCAL = true, bool GEN = false>
__global__ void __launch_bounds__((NW + (COOP ? 0 : 1)) * 32) sw_fill16_kernel(const __grid_constant__ FillArgs a)
{
    using F = Fill16<NW, W, NS, SPLIT, LOCAL>;
    constexpr int ALPHA = F::ALPHA;
    constexpr int BH = F::BH, SKEW = F::SKEW, STEPS = F::STEPS;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int2 *rings = reinterpret_cast<int2 *>(smem_raw);
    uint32_t *selr = reinterpret_cast<uint32_t *>(rings + (NW + 1) * F::RS);
    uint32_t *crings = selr + 2 * F::HALF;
    int *saves = reinterpret_cast<int *>(crings + NW * W);
    uint2 *spbuf = reinterpret_cast<uint2 *>(saves + F::NSAVE * 32 * NW);  // SPM 3 staging, F::SPB per warp
    __shared__ int s_band, s_abort;

    const int warp = threadIdx.x >> 5, lane = lane_id();
    const uint32_t selr_base = (uint32_t)__cvta_generic_to_shared(selr);
    const StripeArgs &S = a.st[blockIdx.x % a.nstripes];
    const int NT = S.NT;
    auto code_at = [&](int col) -> uint32_t {  // 2-bit code of local column col; pad and col < 0: 0
        if (col < 0 || col >= S.w) return 0u;
        const int gc = S.col0 + col;
        return (__ldg(a.B2 + (gc >> 4)) >> ((gc & 15) * 2)) & 3u;
    };
    const bool has_left = S.lb != nullptr, has_right = S.rb != nullptr;
    int bs = 0, bi = LOCAL ? 0 : INT_MAX, bj = LOCAL ? 0 : INT_MAX;
    long long nrep = 0;
    if (*a.err) return;
    StepInfo X;
    X.w = S.w;
    X.hw = LOCAL ? S.w : min(S.w, a.hit_w);
    X.col0 = S.col0;
    X.sp_ld = S.sp_ld;
    X.sp_stride = S.sp_stride;
    X.jcap = S.w - 1;
    X.rbrow = nullptr;
    X.sp_end = S.sp != nullptr ? S.sp + (long long)a.sp_slots * S.sp_stride : nullptr;
    X.sp_span = (long long)a.sp_slots * S.sp_stride;
    // steps at which a lane meets the capture column: low half at k = jcap + 2 lane, high at +1
    const int cap_t0 = X.jcap / STEPS, cap_t1 = (X.jcap + 63) / STEPS;

    for (;;) {
        if (threadIdx.x == 0) {
            int b = atomicAdd(S.ticket, 1) * a.cyc_p + a.cyc_g;
            if (!LOCAL && b > ld_relaxed(a.hit_band)) b = a.nb;
            if (ld_relaxed(a.err)) b = a.nb;
            if (b < a.nb) sp_admit(a, a.row_base + (long long)b * BH, BH);
            s_band = b;
            s_abort = 0;
        }
        __syncthreads();
        const int b = s_band;
        if (b >= a.nb) break;
        const int G = a.band_base + b;           // global band number (progress, colp)
        const int rowtop = a.row_base + b * BH;  // 0-based first row of the band
        if (a.dbg && threadIdx.x == 0 && S.col0 == 0) a.dbg[80 * G] = gtimer();  // debug: band start

        typename F::Lane L;
        const int row0 = rowtop + (warp * 32 + lane) * ALPHA;
        int *sp_ptr = nullptr;
        int sp_r = -1;  // this lane's special row within its strip (-1: none)
        bool warp_sp = false, warp_sp2 = false;
        // a warp with one special lane (SPM 3): its slot, half (row >= NS) and row pointer
        int warp_sps = -1, warp_sphi = 0;
        int band_sps = -1;  // GEN, k >= BH: the slot of the band's one special row (every warp's tile_gen)
        int *warp_spp = nullptr;
        X.rbrow = has_right ? S.rb + row0 + 1 : nullptr;
        auto init_state = [&](bool from_left) {
            // state at the column left of the stripe: the column-0 boundary or the left border
            int tv[ALPHA], ev[ALPHA];
            if (from_left) {
#pragma unroll
                for (int r = 0; r < ALPHA; r++) {
                    const int2 v = ld_sys_int2(S.lb + row0 + 1 + r);
                    tv[r] = v.x;
                    ev[r] = v.y;
                }
            } else if (LOCAL) {
#pragma unroll
                for (int r = 0; r < ALPHA; r++) { tv[r] = -a.gf; ev[r] = -a.gf; }  // E(i,0) := t(i,0), exact
            } else {
                // global: H(i,0) = -(G_open + i G_ext) (reading S9); E(i,0) := t(i,0), exact
#pragma unroll
                for (int r = 0; r < ALPHA; r++) { tv[r] = -(a.go + (row0 + r + 1) * a.ge) - a.gf; ev[r] = tv[r]; }
            }
            int tp;
            if (from_left && row0 > 0) tp = ld_sys_int2(S.lb + row0).x;
            else if (LOCAL || row0 == 0) tp = -a.gf;  // t(0,0): H(0,0) = 0
            else tp = -(a.go + row0 * a.ge) - a.gf;
            L.B = __shfl_sync(0xffffffffu, tv[0], 0);
            L.adj = BIAS16 - L.B;
            L.Bm = L.B - BIAS16;
#pragma unroll
            for (int s = 0; s < NS; s++) {
                L.e[s] = pk(F::tofr(L, ev[s]), F::tofr(L, ev[s + NS]));
                L.t[s] = pk(F::tofr(L, tv[s]), F::tofr(L, tv[s + NS]));
            }
            L.tprev = pk(F::tofr(L, tp), F::tofr(L, tp));
            L.fn = L.t[NS - 1];  // only feeds the high half at column -1 (kept by GUARD)
            const int fl = LOCAL ? min(max(BIAS16 - L.B, 0), 0xffff) : 0;
            L.FL = (uint32_t)fl * 0x10001u;
        };
        if (warp < NW) {
            if constexpr (ALPHA % 16 == 0) {
                // row r's code: bits 2 (r & 15) of word r >> 4 (row0 is a multiple of 16)
                uint32_t wv[ALPHA / 16];
#pragma unroll
                for (int q = 0; q < ALPHA / 16; q++) wv[q] = row0 + 16 * q < a.m ? a.A2[(row0 >> 4) + q] : 0u;
#pragma unroll
                for (int s = 0; s < NS; s++) {
                    const int rp = s, rq = s + NS;
                    L.P[s] = (row0 + rp < a.m) ? a.prof[(wv[rp >> 4] >> (2 * (rp & 15))) & 3u] : PADPROF;
                    L.Q[s] = (row0 + rq < a.m) ? a.prof[(wv[rq >> 4] >> (2 * (rq & 15))) & 3u] : PADPROF;
                }
            } else {
                // alpha 30: strips straddle the 16-code words; one word per row
                auto code_row = [&](int r) -> uint32_t { return (a.A2[r >> 4] >> (2 * (r & 15))) & 3u; };
#pragma unroll
                for (int s = 0; s < NS; s++) {
                    const int rp = row0 + s, rq = row0 + s + NS;
                    L.P[s] = rp < a.m ? a.prof[code_row(rp)] : PADPROF;
                    L.Q[s] = rq < a.m ? a.prof[code_row(rq)] : PADPROF;
                }
            }
            init_state(false);
            if (a.k > 0) {
                // this lane's special row among rows row0 + 1 .. row0 + ALPHA (k >= ALPHA:
                // at most one; the band's bottom row is the I/O warp's drain)
                const int row = ((row0 + a.k) / a.k) * a.k;  // the first multiple of k above row0
                if (row <= row0 + ALPHA && row <= a.m && row != rowtop + BH) {
                    sp_r = row - row0 - 1;
                    sp_ptr = sp_row(a, S, row / a.k - 1);
                }
            }
            warp_sp = __any_sync(0xffffffffu, sp_r >= 0);
            warp_sp2 = GEN && !SPLIT && __any_sync(0xffffffffu, sp_r >= 0 && sp_r != ALPHA - 1);
            warp_sps = -1;
            X.splane = -1;
            band_sps = -1;
            if (GEN && !SPLIT && a.k >= BH) {
                // k >= BH: at most one special row inside the band (its bottom row is
                // the I/O warp's): every warp runs the staged tiles of its slot, so
                // the SM keeps one hot loop (only the owning lane stores)
                const long long row = (((long long)rowtop + a.k) / a.k) * a.k;
                if (row < (long long)rowtop + BH && row <= a.m) {
                    const int r = (int)(row - rowtop - 1) % ALPHA;
                    band_sps = r < NS ? r : r - NS;
                }
            }
            if (GEN && warp_sp && !SPLIT) {
                const unsigned bal = __ballot_sync(0xffffffffu, sp_r >= 0);
                if (__popc(bal) == 1) {  // k >= 32 alpha: one lane (SPM 3)
                    const int sl = __ffs(bal) - 1;
                    const int r = __shfl_sync(0xffffffffu, sp_r, sl);
                    warp_sps = r < NS ? r : r - NS;
                    warp_sphi = r < NS ? 0 : 1;
                    warp_spp = reinterpret_cast<int *>(__shfl_sync(0xffffffffu, reinterpret_cast<unsigned long long>(sp_ptr), sl));
                    X.splane = sl;
                    X.spb = (uint32_t)__cvta_generic_to_shared(spbuf + warp * F::SPB);
                }
            }
        }

        auto io_load = [&](int c) {
            const int need = min((c + 1) * W, NT * W - SKEW);
            if (rowtop > 0) {
                if (lane == 0) {
                    const unsigned long long t0 = gtimer();
                    unsigned long long spins = 0;
                    const unsigned long long want = ptag(a.pepoch, need);
                    while (ld_acquire_u64(S.prog_in + G, a.cross) < want) {
                        if (!LOCAL && ld_relaxed(a.hit_band) < b) { s_abort = 1; break; }
                        if (gtimer() - t0 > (unsigned long long)a.timeout_ns) { atomicExch(a.err, 2); s_abort = 1; break; }
                        __nanosleep(64);
                        spins++;
                    }
                    if (a.dbg && S.col0 == 0 && spins) {  // debug: total wait ns, spin loops, waits
                        a.dbg[80 * G + 5] += gtimer() - t0;
                        a.dbg[80 * G + 6] += spins;
                        a.dbg[80 * G + 7] += 1;
                    }
                    if (a.dbg && S.col0 == 0 && c == 0) {  // debug: tile 0's border wait
                        a.dbg[80 * G + 2] = gtimer();
                        a.dbg[80 * G + 3] = ld_acquire_u64(S.prog_in + G, a.cross) & 0xffffffffull;
                        a.dbg[80 * G + 4] = spins;
                    }
                }
                __syncwarp();
            }
#pragma unroll
            for (int x = lane; x < W; x += 32) {
                const int col = c * W + x;
                rings[F::ridx(col)] = (rowtop == 0) ? top_boundary<LOCAL>(a, S.col0 + col) : __ldcg(S.rowb_in + col);
                // pad columns: code 0 (harmless, see header)
                F::put_sel(selr, col, code_at(col), code_at(col - 1));
            }
        };
        int *io_sp = nullptr;
        if (a.k > 0) {
            const int bottom = rowtop + BH;
            if (bottom <= a.m && bottom % a.k == 0) io_sp = sp_row(a, S, bottom / a.k - 1);
        }
        unsigned int *const colp = band_has_special(rowtop, BH, a.m, a.k) ? S.colp : nullptr;
        auto io_drain = [&](int cd) {
            const int2 *ringN = rings + NW * F::RS;
#pragma unroll
            for (int x = lane; x < W; x += 32) {
                const int col = cd * W - SKEW + x;
                if (col >= 0) {
                    const int2 v = ringN[F::ridx(col)];
                    __stcg(S.rowb_out + col, v);
                    if (io_sp != nullptr && col < S.w) {
                        __stcg(io_sp + col, v.x + a.gf);  // H = t + G_first
                        __stcg(io_sp + S.sp_ld + col, v.y);
                    }
                }
            }
            __threadfence();
            __syncwarp();
            if (lane == 0) {
                publish_progress(a, S, G, cd * W + W - SKEW);
                publish_cols(colp, G, cd, cd * W + W - SKEW);
            }
        };
        auto wait_left = [&]() {
            if (lane == 0) {
                const int fi = b * NW + warp;
                const unsigned long long t0 = gtimer();
                while (ld_acquire_sys(S.lready + fi) != a.epoch || (fi > 0 && ld_acquire_sys(S.lready + fi - 1) != a.epoch)) {
                    if (gtimer() - t0 > (unsigned long long)a.timeout_ns) { atomicExch(a.err, 2); break; }
                    __nanosleep(64);
                }
            }
            __syncwarp();
        };

        // cooperative I/O: this warp's share of each tile's columns
        constexpr int CPW = COOP ? W / NW : W;
        static_assert(!COOP || (W % NW == 0 && W / NW <= 32), "W must split over the warps");
        auto coop_wait = [&](int c) {
            const int need = min((c + 1) * W, NT * W - SKEW);
            if (rowtop > 0 && lane == 0) {
                const unsigned long long t0 = gtimer();
                const unsigned long long want = ptag(a.pepoch, need);
                while (ld_acquire_u64(S.prog_in + G, a.cross) < want) {
                    if (gtimer() - t0 > (unsigned long long)a.timeout_ns) { atomicExch(a.err, 2); s_abort = 1; break; }
                    __nanosleep(64);
                }
            }
            __syncwarp();
        };
        auto coop_fetch = [&](int c, int2 &v, uint32_t &code) {  // issue the loads (results used after compute)
            const int col = c * W + warp * CPW + lane;
            v = (rowtop == 0) ? top_boundary<LOCAL>(a, S.col0 + col) : __ldcg(S.rowb_in + col);
            code = code_at(col) | (code_at(col - 1) << 2);
        };
        auto coop_put = [&](int c, int2 v, uint32_t code) {
            const int col = c * W + warp * CPW + lane;
            rings[F::ridx(col)] = v;
            F::put_sel(selr, col, code & 3u, code >> 2);
        };
        auto coop_drain = [&](int cd) {
            const int col = cd * W - SKEW + warp * CPW + lane;
            if (col >= 0) {
                const int2 v = rings[NW * F::RS + F::ridx(col)];
                __stcg(S.rowb_out + col, v);
                if (io_sp != nullptr && col < S.w) {
                    __stcg(io_sp + col, v.x + a.gf);
                    __stcg(io_sp + S.sp_ld + col, v.y);
                }
                __threadfence();
            }
        };

        if constexpr (COOP) {
            coop_wait(0);
            if (lane < CPW) {
                int2 v;
                uint32_t code;
                coop_fetch(0, v, code);
                coop_put(0, v, code);
            }
        } else {
            if (warp == NW) io_load(0);
        }
        __syncthreads();
        const int S_END = NT + 2 * (NW - 1);
        int *sv = saves + warp * F::NSAVE * 32;
        for (int s = 0; s < S_END + 1; ++s) {
            int2 fv = make_int2(0, 0);
            uint32_t fcode = 0u;
            if constexpr (COOP) {
                if (s + 1 < NT) {
                    coop_wait(s + 1);
                    if (lane < CPW) coop_fetch(s + 1, fv, fcode);
                }
            }
            if (warp < NW) {
                const int c = s - 2 * warp;
                if (c >= 0 && c < NT) {
                    const uint32_t rin = pin((uint32_t)__cvta_generic_to_shared(crings + warp * W));
                    const uint32_t rout = pin((uint32_t)__cvta_generic_to_shared(rings + (warp + 1) * F::RS));
                    const uint32_t selr_s = pin(selr_base);
                    if (c == 0 && has_left) {
                        wait_left();
                        init_state(true);
                    }
                    if (c > 0) F::rebase(a, L);
                    F::convert_ring(a, L, rings + warp * F::RS, crings + warp * W, c, lane);
                    // the running best of all CTAs: loaded here, used after the tile
                    // (so the L2 round trip overlaps the tile instead of stalling it)
                    const int gbest = LOCAL ? ld_relaxed(a.gbest) : 0;
                    const int bs0 = bs;
                    F::save(L, sv, lane);
                    uint32_t tm;
                    const bool cap = has_right && c >= cap_t0 && c <= cap_t1;
                    if (cap) {
                        tm = (GEN && warp_sps >= 0) ? F::template tile<true, false, 3, true>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r)
                           : warp_sp2 ? F::template tile<true, false, GEN ? 2 : 1, true>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r)
                           : warp_sp ? F::template tile<true, false, 1, true>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r)
                                     : F::template tile<true, false, 0, true>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r);
                        if (c == cap_t1) {
                            __threadfence_system();
                            __syncwarp();
                            if (lane == 0 && S.rready != nullptr) st_release_sys_s32(S.rready + b * NW + warp, a.epoch);
                        }
                    } else if (c == 0) {
                        tm = (GEN && warp_sps >= 0) ? F::template tile<true, false, 3, false>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r)
                           : warp_sp2 ? F::template tile<true, false, GEN ? 2 : 1, false>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r)
                           : warp_sp ? F::template tile<true, false, 1, false>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r)
                                     : F::template tile<true, false, 0, false>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r);
                    } else if (GEN && (band_sps >= 0 || warp_sps >= 0)) {
                        // one special lane: staged (SPM 3), the slot a compile-time constant
                        tm = F::tile_gen(band_sps >= 0 ? band_sps : warp_sps, a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r);
                    } else if (warp_sp2) {
                        tm = F::template tile<false, false, GEN ? 2 : 1, false>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r);
                    } else if (warp_sp) {
                        tm = F::template tile<false, false, 1, false>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, sp_r);
                    } else {
                        tm = F::template tile<false, false, 0, false>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, nullptr, -1);
                    }
                    const int tmax = F::toabs(L, max(lo16(tm), hi16(tm))) + F::tmax_off(a);
                    const int thr = LOCAL ? max(max(bs0, gbest), 1) : a.goal;
                    if (__any_sync(0xffffffffu, tmax >= thr)) {
                        F::restore(L, sv, lane);
                        const int obs = bs, obi = bi, obj = bj;
                        F::template tile<true, true, 0, false>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, nullptr, -1);
                        if (lane == 0) nrep++;
                        if (LOCAL) {
                            if (bs > obs) atomicMax(a.gbest, bs);
                        } else if (bi != obi || bj != obj) {
                            atomicMin(a.hit_key, ((unsigned long long)(unsigned)bi << 32) | (unsigned)bj);
                            atomicMin(a.hit_band, b);
                        }
                    }
                    if (GEN && warp_sps >= 0) {
                        // SPM 3: the special lane's columns of this tile (staged
                        // in the tile's frame), coalesced
                        __syncwarp();
#pragma unroll
                        for (int x = lane; x < STEPS; x += 32) {
                            const int jl = c * STEPS + x - 2 * X.splane, col = jl - warp_sphi;
                            if (col >= 0 && col < X.w) {
                                const uint2 v = spbuf[warp * F::SPB + (jl & (F::SPB - 1))];
                                __stcg(warp_spp + col, F::toabs(L, warp_sphi ? hi16(v.x) : lo16(v.x)) + a.gf);  // H = t + G_first
                                __stcg(warp_spp + X.sp_ld + col, F::toabs(L, warp_sphi ? hi16(v.y) : lo16(v.y)));
                            }
                        }
                    }
                }
            } else {
                if (s + 1 < NT) io_load(s + 1);
                const int cd = s - 1 - 2 * (NW - 1);
                if (cd >= 0) io_drain(cd);
                if (!LOCAL && lane == 0 && ld_relaxed(a.hit_band) < b) s_abort = 1;
            }
            const int cdc = s - 1 - 2 * (NW - 1);
            if constexpr (COOP) {
                if (lane < CPW) {
                    if (s + 1 < NT) coop_put(s + 1, fv, fcode);
                    if (cdc >= 0) coop_drain(cdc);
                }
            }
            __syncthreads();
            if constexpr (COOP) {
                // every warp's drain of tile cdc is stored and fenced: publish it
                if (threadIdx.x == 0 && cdc >= 0 && !s_abort) {
                    publish_progress(a, S, G, cdc * W + W - SKEW);
                    publish_cols(colp, G, cdc, cdc * W + W - SKEW);
                }
            }
            if (s_abort) break;
        }
        if (threadIdx.x == (COOP ? 0 : NW * 32) && !s_abort) publish_progress(a, S, G, INT_MAX);
        if (a.dbg && threadIdx.x == 0 && S.col0 == 0) a.dbg[80 * G + 15] = gtimer();  // debug: band end
        if constexpr (!LOCAL) {
            if (a.match && !s_abort) {
                // Stage-2 goal-based matching, as in the
                // int32 kernel: the capture tiles left (t, E) of the special row's DP
                // column for every row of the band in S.rb (int32, absolute); row j'
                // is original column j = j_c - j', t + G_first the reverse H there,
                // E the reverse F.  Once per band, coalesced.
                __syncthreads();
                unsigned long long key = ~0ull;
                const int hi = min(rowtop + BH, a.m);
                for (int row = rowtop + 1 + (int)threadIdx.x; row <= hi; row += (int)blockDim.x) {
                    const int2 v = __ldcg(S.rb + row);
                    const int j = a.mjc - row;
                    const long long hs = (a.mH != nullptr && j > 0) ? (long long)__ldg(a.mH + j - 1) : 0ll;
                    const long long fs = (a.mH != nullptr && j > 0) ? (long long)__ldg(a.mF + j - 1) : (long long)NEG;
                    int kind = -1;
                    if (hs + v.x + a.gf == a.goal) kind = 0;                                          // H junction
                    else if (fs > NEG / 2 && v.y > NEG / 2 && fs + v.y + a.go == a.goal) kind = 1;  // gap junction (S18)
                    if (kind >= 0) key = min(key, ((unsigned long long)(unsigned)row << 32) | (unsigned)(S.w + kind));
                }
                if (key != ~0ull) {
                    atomicMin(a.hit_key, key);
                    atomicMin(a.hit_band, b);
                }
            }
        }
        if (a.k > 0) {
            __threadfence();
            __syncthreads();
            if (threadIdx.x == 0) {
                const long long lo = (long long)rowtop + 1, hi = min((long long)rowtop + BH, (long long)a.m);
                long long q = (lo + a.k - 1) / a.k;
                if (q * a.k <= hi) {
                    __threadfence_system();
                    for (; q * a.k <= hi; q++) st_release_sys(S.row_done + (q - 1), 1u);
                }
            }
        }
    }

    if (lane == 0 && nrep) atomicAdd(a.replays, (unsigned long long)nrep);
    if constexpr (LOCAL) {  // global: the hits went to hit_key / hit_band
        __shared__ int4 red[NW + 1];
        for (int o = 16; o > 0; o >>= 1) {
            const int s2 = __shfl_down_sync(0xffffffffu, bs, o);
            const int i2 = __shfl_down_sync(0xffffffffu, bi, o);
            const int j2 = __shfl_down_sync(0xffffffffu, bj, o);
            if (better(s2, i2, j2, bs, bi, bj)) { bs = s2; bi = i2; bj = j2; }
        }
        if (lane == 0) red[warp] = make_int4(bs, bi, bj, 0);
        __syncthreads();
        if (threadIdx.x == 0) {
            int4 r = make_int4(0, 0, 0, 0);
            for (int w = 0; w < NW; w++)
                if (red[w].x > 0 && better(red[w].x, red[w].y, red[w].z, r.x, r.y, r.z)) r = red[w];
            a.slots[blockIdx.x] = r;
        }
    }
}

}  // namespace swb
