// sw_fill.cuh -- sm_100a Stage-1 / reverse-pass matrix fill (CUDAlign 2.0,
// Sandes & de Melo IPDPS 2011; P:<line> = /root/reference/PAPER.md line).
//
// What one launch computes: the Smith-Waterman/Gotoh recurrences Eq. 1-3
// over all m x n cells in linear space, the best score with its
// exact (min i, min j) end cell, and every k-th special row of
// (H, F); or, in GLOBAL mode, the anchored global recurrence of
// the reverse pass and its first cell equal to `goal`.
//
// B200 design (the paper's GT200 external-diagonal
// launches, short/long phases and shifted bus are replaced):
//  * Band = BH = ALPHA*32*NW consecutive rows.  One persistent CTA takes a band
//    from an atomic ticket and sweeps ALL columns of it left to right; bands
//    are taken in order, so a CTA only ever waits on a band owned by a running
//    CTA (deadlock-free with any grid size).
//  * Lane = ALPHA consecutive rows whose (E, t = H - G_first) live in
//    registers; the substitution score p(i,j)+G_first for the lane's rows is a
//    per-row int8x4 "profile" word selected with one PRMT per cell by the
//    column's 2-bit code.  A lane handles TWO columns per step, the second one
//    row behind the first, so its vertical dependency chain (F -> H -> t ->
//    next row) runs as two interleaved chains (ILP 2).  Lanes of a warp form
//    a wavefront skewed by two columns; (t, F) of a lane's bottom row passes
//    to the next lane by SHFL, to the next warp through a shared-memory ring,
//    to the next band through the row border in global memory (in place,
//    n x 8 B), gated by a per-band progress counter (release/acquire, gpu).
//  * Warps of a CTA are skewed by 2 tiles of W columns and advance in lockstep
//    intervals separated by __syncthreads.  A dedicated I/O warp loads the top
//    border and column codes one tile ahead and drains the bottom row one tile
//    behind, publishing progress.
//  * Best cell: a per-tile maximum (cheap); a warp replays a tile with exact
//    (score, i, j) tracking only when some lane's tile maximum reaches the
//    running threshold max(own best, global best hint, 1).  Any cell equal to
//    the final best is therefore replayed, so the reported cell is exact.
#pragma once
#include <cstdint>
#include <climits>
#include <cuda_runtime.h>

namespace swb {

constexpr int NEG = -(1 << 30);            // E(i,0), F(0,j) = "-infinity" (reading S3)
constexpr uint32_t PADPROF = 0x80808080u;  // profile of padding rows / padding column: -128
constexpr int LANE_SKEW = 2;               // columns per lane step

constexpr int MAX_STRIPES = 8;

// One column stripe [col0, col0 + w) of the matrix.  A launch
// runs nstripes stripes (CTA -> stripe = blockIdx.x % nstripes): 1 per GPU in
// the multi-GPU column-stripe pipeline, several "virtual" stripes on one GPU
// for testing.
//
// Band addressing: a launch runs the bands b = t * cyc_p +
// cyc_g (t = 0, 1, ... its ticket) of one SEGMENT of rows: b < nb, first DP
// row row_base + b * BH (0-based), global band number G = band_base + b.
// Band G reads its top border from rowb_in gated by prog_in[G] and drains its
// bottom row into rowb_out, publishing prog_out[G + 1].  One GPU, one
// segment: rowb_in == rowb_out (in place) and prog_in == prog_out.  Band-cyclic
// multi-GPU: rowb_out / prog_out are the NEXT GPU's rowb_in / prog_in (peer
// memory over NVLink).  A tail segment (a second launch with a smaller band
// height for the last partial wave) continues the same arrays.  Progress words
// are epoch-tagged, (epoch << 32) | columns, so they never need re-zeroing.
struct StripeArgs {
    int col0;            // first global 0-based column
    int w;               // real columns of the stripe
    int ncols_pad;       // w rounded up to a multiple of W
    int NT;              // tiles each warp runs per band = ncols_pad / W + ceil(lane skew / W)
    const int2 *rowb_in; // row border read by this launch's bands: (t, F) per local column, >= NT*W + W entries
    int2 *rowb_out;      // row border written by the drain (== rowb_in on one GPU)
    const unsigned long long *prog_in;  // [G]: columns of band G-1's bottom row published (epoch-tagged)
    unsigned long long *prog_out;       // [G + 1] written by band G
    int *ticket;         // band ticket of this stripe
    int *sp;             // special-row ring (this stripe's slice): row q at slot q % sp_slots: H, then F at + sp_ld
    long long sp_stride;
    int sp_ld;
    unsigned int *row_done;  // mapped host flags, one per special row
    unsigned int *colp;  // mapped host words, one per global band: leading columns of the band's special rows that are final
    const int2 *lb;      // left border (t, E) per DP row 0..m at column col0 - 1 (null: column-0 boundary)
    const int *lready;   // per (band, warp) epoch flags guarding lb
    int2 *rb;            // right neighbour's lb (null: last stripe); a peer-GPU pointer across GPUs
    int *rready;         // right neighbour's lready
};

struct FillArgs {
    int m;               // rows of S0
    int n;               // columns of S1 (all stripes)
    int nb;              // bands of this launch's segment (band b covers rows row_base + b BH + 1 ..)
    int row_base;        // 0-based first row of the segment (0 unless a tail segment)
    int band_base;       // global band number of the segment's band 0
    int cyc_p, cyc_g;    // band-cyclic multi-GPU: this GPU runs bands b = t * cyc_p + cyc_g (1, 0 on one GPU)
    int cross;           // 1: the row border / progress go to another GPU (system-scope release)
    int sp_slots;        // special-row ring slots R (>= the rows of one band)
    const unsigned long long *sp_released;  // mapped host counter: rows 0 .. value-1 have left the ring
    unsigned admit_ns;   // poll interval of the ring admission
    int go, ge, gf;      // G_open, G_ext, G_first = go + ge
    int one;             // always 1 (see imad())
    uint32_t prof[4];    // profile word for row code a: byte x = (a == x ? ma : mi) + gf
    int pm_gf, pn_gf;    // WIDE kernels: match + gf, mismatch + gf (any scoring within the SW_ERANGE rule)
    const uint32_t *A2;  // S0 codes, 2 bits each, 16 per word
    const uint32_t *B2;  // S1 codes (global columns)
    int *err;            // non-zero: encode found a bad byte -> do nothing; kernel sets 2 on a wait timeout
    int k;               // special-row interval (0 = none)
    int *gbest;          // running best-score hint
    int4 *slots;         // per-CTA (score, i, j, 0)
    int goal;            // GLOBAL mode
    int hit_w;           // GLOBAL: DP columns 1..hit_w may hold a goal hit (start check)
    int anchor_gap;      // GLOBAL: the anchor is a gap crosspoint: column 0 and the corner diagonal are -inf (S20)
    int match;           // Stage-2 matching at the last column of a transposed partition
    int mjc;             // anchor column j_c: DP row j' of the partition is original column j_c - j'
    const int *mH, *mF;  // special row r's H and F at original columns 1..n (index j - 1); null: row 0 (H 0, F -inf)
    unsigned long long *hit_key;  // min over hits of (i' << 32 | j')
    int *hit_band;       // min band containing a hit
    unsigned long long *replays;
    int epoch;           // value written to the column-stripe border flags by this call
    int pepoch;          // tag of this call's band-progress words (strictly increasing per progress array)
    long long timeout_ns;  // spin-wait watchdog
    int nstripes;
    int force_slow;      // unused
    unsigned long long *dbg;  // optional: per band 80 x %globaltimer; slot 0 band start, 1 first tile, 15 band end
    StripeArgs st[MAX_STRIPES];
};

// Per-CTA view of the stripe fields the cell step needs.
struct StepInfo {
    int w;               // stripe width (pad columns are >= w)
    int col0;            // global column of local column 0
    int sp_ld;
    long long sp_stride;
    int *sp_end;         // end of the special-row ring: the slot after the last wraps to the first
    long long sp_span;   // sp_slots * sp_stride
    int jcap;            // local column whose (t, E) goes to the right neighbour
    int2 *rbrow;         // right-border destination for this lane's first row
    int hw;              // columns eligible for tracking (w, or the Stage-2 start-check width)
    int splane;          // packed GEN kernel, SPM 3: the warp's one lane with a special row
    uint32_t spb;        // ... and the warp's staging buffer (shared, 128 x uint2) for it
};

__device__ __forceinline__ unsigned long long gtimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t) : : "memory");  // ordered with barriers (debug stamps)
    return t;
}

__device__ __forceinline__ uint32_t col_sel(uint32_t code)  // code 0..3, 4 = pad
{
    const uint32_t s = code | 8u;  // PRMT: bit 3 of a selector nibble replicates the sign
    return code | (s << 4) | (s << 8) | (s << 12);
}

__device__ __forceinline__ int prmt(uint32_t a, uint32_t b, uint32_t sel)
{
    int r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
    return r;
}

// Shared-memory accesses through 32-bit shared-window addresses (kept in
// registers; avoids re-deriving the generic window inside the hot loop).
__device__ __forceinline__ int4 lds_v4(uint32_t addr)
{
    int4 v;
    asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr) : "memory");
    return v;
}
__device__ __forceinline__ uint2 lds_v2u(uint32_t addr)
{
    uint2 v;
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(addr) : "memory");
    return v;
}
__device__ __forceinline__ void sts_v4(uint32_t addr, int4 v)
{
    asm volatile("st.shared.v4.s32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
// An opaque copy: the result cannot be rematerialised by the compiler, so a
// value computed once outside a loop stays in a register inside it.
__device__ __forceinline__ uint32_t pin(uint32_t x)
{
    uint32_t y;
    asm volatile("mov.b32 %0, %1;" : "=r"(y) : "r"(x));
    return y;
}
__device__ __forceinline__ int lane_id()
{
    int l;
    asm volatile("mov.u32 %0, %%laneid;" : "=r"(l));
    return l;
}

// -G_ext and -G_first of the int32 cell update: instruction immediates in the
// patched image (sw_fill16_patch.cu, SWB_PATCH), kernel arguments otherwise.
#ifndef SWB_I32MODE
#define SWB_I32MODE 0  // int32 cell update: 0 = H form (default, measured faster), 1 = D form
#endif
#ifndef SWB_K_NGE1
#define SWB_K_NGE1 0x2ae8944au
#define SWB_K_NGF1 0x625558ecu
#endif
#ifdef SWB_PATCH
#define NGE(a) ((int)SWB_K_NGE1)
#define NGF(a) ((int)SWB_K_NGF1)
#else
#define NGE(a) (-(a).ge)
#define NGF(a) (-(a).gf)
#endif

// x * one + y through the FMA pipe (IMAD); `one` is a runtime 1 so ptxas
// cannot fold the add into an ALU-pipe VIADDMNMX.
__device__ __forceinline__ int imad(int x, int one, int y)
{
    int r;
    asm("mad.lo.s32 %0, %1, %2, %3;" : "=r"(r) : "r"(x), "r"(one), "r"(y));
    return r;
}

__device__ __forceinline__ int ld_acquire(const int *p)
{
    int v;
    asm volatile("ld.acquire.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ int ld_relaxed(const int *p)
{
    int v;
    asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(int *p, int v)
{
    asm volatile("st.release.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_sys(unsigned int *p, unsigned int v)
{
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Epoch-tagged band progress: a word from an earlier call is
// smaller than every tag of this call, so the arrays are never re-zeroed.
__device__ __forceinline__ unsigned long long ptag(int epoch, int cols)
{
    return ((unsigned long long)(unsigned)epoch << 32) | (unsigned)cols;
}
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long *p, int sys)
{
    unsigned long long v;
    if (sys) asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    else asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u64(unsigned long long *p, unsigned long long v, int sys)
{
    if (sys) asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
    else asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// Publish `cols` leading columns of band G's bottom row (after its stores are fenced).
__device__ __forceinline__ void publish_progress(const FillArgs &a, const StripeArgs &S, int G, int cols)
{
    cols = max(cols, 0);  // the first drained tile of a W = 32 kernel publishes W - SKEW < 0 columns
    if (a.cross) __threadfence_system();
    st_release_u64(S.prog_out + G + 1, ptag(a.pepoch, cols), a.cross);
}
// Ring slot of special row q (0-based: DP row (q + 1) k).
__device__ __forceinline__ int *sp_row(const FillArgs &a, const StripeArgs &S, long long q)
{
    return S.sp + (q % a.sp_slots) * S.sp_stride;
}
#ifndef SWB_ADMIT_POLL
#define SWB_ADMIT_POLL 1
#endif
// Back-pressure of the special-row ring (P:178's bounded SRA): before a band
// with rows [lo, hi] starts, the rows that used its slots before must have left
// the device: released >= q_hi - R + 1 (deadlock-free: R >= the rows of one
// band, and the rows waited for belong to earlier bands).  Thread 0 only.
__device__ __forceinline__ void sp_admit(const FillArgs &a, long long rowtop, int BH)
{
    if (a.k <= 0 || a.sp_released == nullptr) return;
    const long long hi = min(rowtop + BH, (long long)a.m);
    const long long q_hi = hi / a.k - 1;
    if (q_hi < 0 || (q_hi + 1) * a.k <= rowtop) return;  // no special row in the band
    const unsigned long long need = (unsigned long long)max(0ll, q_hi - a.sp_slots + 1);
    if (need == 0) return;
    const unsigned long long t0 = gtimer();
    while (true) {
        unsigned long long v;
#if SWB_ADMIT_POLL == 0
        asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(a.sp_released) : "memory");
#else
        asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(a.sp_released) : "memory");
#endif
        if (v >= need) break;
        if (gtimer() - t0 > 4ull * (unsigned long long)a.timeout_ns) { atomicExch(a.err, 2); break; }
        __nanosleep(a.admit_ns);
    }
    __threadfence_system();
}

// True when DP rows rowtop+1 .. min(rowtop+BH, m) hold a special row (k > 0).
__device__ __forceinline__ bool band_has_special(long long rowtop, int BH, int m, int k)
{
    if (k <= 0) return false;
    const long long lo = rowtop + 1, hi = min(rowtop + BH, (long long)m);
    return ((lo + k - 1) / k) * k <= hi;
}

// Every 16th drained tile of a band holding special rows: tell the host how
// many leading columns of them are final, so it can copy them while the band
// is still running (the rows of a one-wave matrix all complete at the end).
// Called by the thread that published the band's progress, after the drained
// stores of the whole warp/CTA are fenced.
__device__ __forceinline__ void publish_cols(unsigned int *colp, int b, int cd, int cols)
{
    if (colp != nullptr && (cd & 15) == 15) {
        __threadfence_system();
        st_release_sys(colp + b, (unsigned int)cols);
    }
}

// (score, i, j) total order: higher score, then smaller i, then smaller j (reading S4)
__device__ __forceinline__ bool better(int s, int i, int j, int bs, int bi, int bj)
{
    return s > bs || (s == bs && (i < bi || (i == bi && j < bj)));
}

template <int W, int NW>
struct Smem {
    // warp lag in tiles: lane 31 of the warp above must be done with a tile's
    // columns before lane 0 below starts them (1 + ceil(skew / W), skew <= 63)
    static constexpr int LAG = 1 + (63 + W - 1) / W;
    static constexpr int RING = W >= 64 ? 4 * W : 256;
    static constexpr int SRING_MIN = (LAG * (NW - 1) + 2) * W + 64;
    static constexpr int SRING = SRING_MIN <= 256 ? 256 : SRING_MIN <= 512 ? 512 : SRING_MIN <= 1024 ? 1024 : SRING_MIN <= 2048 ? 2048 : 4096;
};

// WIDE = true: the substitution score p + G_first is selected from the two
// int32 values (pm_gf, pn_gf) by comparing the row's and the column's 2-bit
// codes (ISETP + SEL) instead of a PRMT of the int8x4 profile, so any scoring
// inside the SW_ERANGE rule runs (|p + G_first| > 127 included).  Pad rows and
// pad columns get codes that never match: their cells are real-looking
// mismatches, which is harmless -- they lie below / right of every real cell
// and the exact tracking ignores rows > m and columns > w.
template <int ALPHA, int NW, int W, bool LOCAL, bool WIDE = false>
struct Fill {
    static constexpr int BH = ALPHA * 32 * NW;
    static constexpr int RING = Smem<W, NW>::RING;
    static constexpr int SRING = Smem<W, NW>::SRING;
    static constexpr int NSAVE = 2 * ALPHA + 5;
    static constexpr int SKEW = 31 * LANE_SKEW;  // columns lane 31 lags lane 0
    static constexpr int STEPS = W / LANE_SKEW;  // lane steps per tile
    static constexpr int LAG = 1 + (SKEW + W - 1) / W;  // tiles warp w+1 trails warp w
    static constexpr int GUARD_TILES = (31 + STEPS - 1) / STEPS;  // tiles where some lane is left of column 0
    static_assert(W % 32 == 0 && LAG <= Smem<W, NW>::LAG, "W multiple of 32");
    static_assert((LAG + 1) * W <= RING, "ring holds the producer/consumer span");
    static_assert(ALPHA % 2 == 0 && ALPHA <= 16, "ALPHA even, <= 16");

    static size_t smem_bytes()
    {
        return sizeof(int2) * RING * (NW + 1) + sizeof(uint32_t) * SRING + sizeof(int) * NSAVE * 32 * NW;
    }

    static __device__ __forceinline__ int subst(const FillArgs &a, uint32_t P, uint32_t sel)
    {
        if constexpr (WIDE) return P == sel ? a.pm_gf : a.pn_gf;
        else return prmt(P, PADPROF, sel);
    }

    // ---------------------------------------------------------------- per-lane state
    struct Lane {
        uint32_t P[ALPHA];
        int e[ALPHA];      // E(r, j-1) of the last column done
        int t[ALPHA];      // t = H - G_first at (r, j-1)
        int tprev;         // t of the row above this strip at the last column done (diagonal input)
        int out_t0, out_f0, out_t1, out_f1;  // (t, F) of the strip's bottom row at the two last columns
    };

    // One lane step (warp-synchronous): the lane handles 0-based columns
    // j0 = 2 (k - lane) and j0 + 1.  TRACK: exact best / first-hit tracking.
    // SPM: 0 = no special rows, 1 = special rows are strip-bottom rows,
    // 2 = special rows anywhere in the strip (bitmask).
    template <bool GUARD, bool TRACK, int SPM, bool CAP = false>
    static __device__ __forceinline__ int step(const FillArgs &a, const StepInfo &X, Lane &L, int k, int lane,
                                               uint32_t ring_in, uint32_t ring_out, uint32_t selr, int tmax,
                                               int row1, int &bs, int &bi, int &bj, int *sp_ptr, uint32_t smask)
    {
        int a_t = __shfl_up_sync(0xffffffffu, L.out_t0, 1);
        int a_f = __shfl_up_sync(0xffffffffu, L.out_f0, 1);
        int b_t = __shfl_up_sync(0xffffffffu, L.out_t1, 1);
        int b_f = __shfl_up_sync(0xffffffffu, L.out_f1, 1);
        const int j0 = LANE_SKEW * (k - lane);
        if (lane == 0) {
            const int4 v = lds_v4(ring_in + (uint32_t)(j0 & (RING - 1)) * 8u);
            a_t = v.x; a_f = v.y; b_t = v.z; b_f = v.w;
        }
        if (GUARD && j0 < 0) return tmax;
        const uint2 sl = lds_v2u(selr + (uint32_t)(j0 & (SRING - 1)) * 4u);
        int tdA = L.tprev;  // t(r0-1, j0-1)
        int tdB = a_t;      // t(r0-1, j0)
        L.tprev = b_t;
#if SWB_I32MODE == 1
        // F of the lane's first row from the row above (t, F): Eq. 3
        int fA = __viaddmax_s32(a_f, NGE(a), a_t), fB = __viaddmax_s32(b_f, NGE(a), b_t);
        int tuA = a_t, fuA = a_f, tuB = b_t, fuB = b_f;
        const int gf = a.gf;
        int *spp = sp_ptr;
#pragma unroll
        for (int r = 0; r < ALPHA; r++) {
            // column j0, with D = max(H_diag + p, E[, 0]) (Eq. 1 without F):
            //   E  = max(E_left - G_ext, t_left)            Eq. 2 (t = H - G_first)
            //   Dg = D - G_first
            //   t  = max(F - G_first, Dg)                    (H = max(D, F), Eq. 1)
            //   F' = max(F - G_ext, Dg)                      Eq. 3 for the next row
            // F' = max(F - G_ext, t) = max(F - G_ext, D - G_first, F - G_first) and
            // G_ext <= G_first, so the chain down the rows is one VIADDMNMX per row;
            // the constants are immediates in the patched image.
            const int eA = __viaddmax_s32(L.e[r], NGE(a), L.t[r]);
            const int pA = subst(a, L.P[r], sl.x);
            const int xA = tdA + pA;
            const int dA = LOCAL ? __vimax_s32_relu(eA, xA) : max(eA, xA);
            const int dgA = dA + NGF(a);
            const int tA = __viaddmax_s32(fA, NGF(a), dgA);
            fuA = fA;  // F of this row
            fA = __viaddmax_s32(fA, NGE(a), dgA);
            tdA = L.t[r];
            tuA = tA;
            // column j0 + 1 (one row behind column j0 in the dependency chain)
            const int eB = __viaddmax_s32(eA, NGE(a), tA);
            const int pB = subst(a, L.P[r], sl.y);
            const int xB = tdB + pB;
            const int dB = LOCAL ? __vimax_s32_relu(eB, xB) : max(eB, xB);
            const int dgB = dB + NGF(a);
            const int tB = __viaddmax_s32(fB, NGF(a), dgB);
            fuB = fB;
            fB = __viaddmax_s32(fB, NGE(a), dgB);
            tdB = tA;
            tuB = tB;
            L.e[r] = eB;
            L.t[r] = tB;
            tmax = __vimax3_s32(tmax, tA, tB);  // the tile maximum of t = H - G_first
            if (SPM == 2 || TRACK) {
                const int hA = tA + gf, hB = tB + gf;
                if (SPM == 2) {
                    if (smask & (1u << r)) {
                        if (j0 < X.w) { spp[j0] = hA; spp[X.sp_ld + j0] = fuA; }
                        if (j0 + 1 < X.w) { spp[j0 + 1] = hB; spp[X.sp_ld + j0 + 1] = fuB; }
                        spp += X.sp_stride;
                        if (spp >= X.sp_end) spp -= X.sp_span;
                    }
                }
                if (TRACK) {
                    const int row = row1 + r;
                    if (row <= a.m) {
                        const int cA = X.col0 + j0 + 1, cB = cA + 1;  // global DP columns
                        if (j0 + 1 <= X.hw) {
                            if (LOCAL) {
                                if (better(hA, row, cA, bs, bi, bj)) { bs = hA; bi = row; bj = cA; }
                            } else if (hA == a.goal && (row < bi || (row == bi && cA < bj))) {
                                bi = row; bj = cA;
                            }
                        }
                        if (j0 + 2 <= X.hw) {
                            if (LOCAL) {
                                if (better(hB, row, cB, bs, bi, bj)) { bs = hB; bi = row; bj = cB; }
                            } else if (hB == a.goal && (row < bi || (row == bi && cB < bj))) {
                                bi = row; bj = cB;
                            }
                        }
                    }
                }
            }
            if (CAP) {  // the stripe's last column: hand (t, E) to the right neighbour
                if (j0 == X.jcap) X.rbrow[r] = make_int2(tA, eA);
                if (j0 + 1 == X.jcap) X.rbrow[r] = make_int2(tB, eB);
            }
        }
#else
        int tuA = a_t, fuA = a_f, tuB = b_t, fuB = b_f;
                const int gf = a.gf;
        int *spp = sp_ptr;
#pragma unroll
        for (int r = 0; r < ALPHA; r++) {
            // column j0: Eq. 2, Eq. 3, Eq. 1 (p' = p + G_first applied to t = H - G_first).
            // Instruction mix balanced over the ALU pipe (DPX max, PRMT) and the
            // FMA pipe (the adds, as IMAD with a runtime 1): DESIGN.md section 5.
            const int eA = __viaddmax_s32(L.e[r], NGE(a), L.t[r]);
            fuA = max(fuA + NGE(a), tuA);
            const int pA = subst(a, L.P[r], sl.x);
            const int xA = tdA + pA;
            const int hA = LOCAL ? __vimax3_s32_relu(eA, fuA, xA) : __vimax3_s32(eA, fuA, xA);
            tdA = L.t[r];
            const int tA = hA + NGF(a);
            tuA = tA;
            // column j0 + 1 (one row behind column j0 in the dependency chain)
            const int eB = __viaddmax_s32(eA, NGE(a), tA);
            fuB = max(fuB + NGE(a), tuB);
            const int pB = subst(a, L.P[r], sl.y);
            const int xB = tdB + pB;
            const int hB = LOCAL ? __vimax3_s32_relu(eB, fuB, xB) : __vimax3_s32(eB, fuB, xB);
            tdB = tA;
            const int tB = hB + NGF(a);
            tuB = tB;
            L.e[r] = eB;
            L.t[r] = tB;
            tmax = __vimax3_s32(tmax, tA, tB);  // tile maximum of t = H - G_first
            if (SPM == 2) {
                if (smask & (1u << r)) {
                    if (j0 < X.w) { spp[j0] = hA; spp[X.sp_ld + j0] = fuA; }
                    if (j0 + 1 < X.w) { spp[j0 + 1] = hB; spp[X.sp_ld + j0 + 1] = fuB; }
                    spp += X.sp_stride;
                        if (spp >= X.sp_end) spp -= X.sp_span;
                }
            }
            if (CAP) {  // the stripe's last column: hand (t, E) to the right neighbour
                if (j0 == X.jcap) X.rbrow[r] = make_int2(tA, eA);
                if (j0 + 1 == X.jcap) X.rbrow[r] = make_int2(tB, eB);
            }
            if (TRACK) {
                const int row = row1 + r;
                if (row <= a.m) {
                    const int cA = X.col0 + j0 + 1, cB = cA + 1;  // global DP columns
                    if (j0 + 1 <= X.hw) {
                        if (LOCAL) {
                            if (better(hA, row, cA, bs, bi, bj)) { bs = hA; bi = row; bj = cA; }
                        } else if (hA == a.goal && (row < bi || (row == bi && cA < bj))) {
                            bi = row; bj = cA;
                        }
                    }
                    if (j0 + 2 <= X.hw) {
                        if (LOCAL) {
                            if (better(hB, row, cB, bs, bi, bj)) { bs = hB; bi = row; bj = cB; }
                        } else if (hB == a.goal && (row < bi || (row == bi && cB < bj))) {
                            bi = row; bj = cB;
                        }
                    }
                }
            }
        }
#endif
        L.out_t0 = tuA; L.out_f0 = fuA;
        L.out_t1 = tuB; L.out_f1 = fuB;
        if (SPM == 1 && sp_ptr != nullptr) {
            if (j0 < X.w) { sp_ptr[j0] = tuA + gf; sp_ptr[X.sp_ld + j0] = fuA; }  // H = t + G_first
            if (j0 + 1 < X.w) { sp_ptr[j0 + 1] = tuB + gf; sp_ptr[X.sp_ld + j0 + 1] = fuB; }
        }
        if (!TRACK && lane == 31) sts_v4(ring_out + (uint32_t)(j0 & (RING - 1)) * 8u, make_int4(tuA, fuA, tuB, fuB));
        return tmax;
    }

    // Rare tiles (tile 0 with its lane guard, exact replays, generic special
    // rows): inlined so the lane state stays in registers, but not unrolled.
    template <bool GUARD, bool TRACK, int SPM, bool CAP = false>
    static __device__ __forceinline__ int tile(const FillArgs &a, const StepInfo &X, Lane &L, int c, int lane,
                                               uint32_t ring_in, uint32_t ring_out, uint32_t selr, int row1,
                                               int &bs, int &bi, int &bj, int *sp_ptr, uint32_t smask)
    {
        int tmax = INT_MIN;
        const int k0 = c * STEPS;
#pragma unroll 1
        for (int kk = 0; kk < STEPS; kk++)
            tmax = step<GUARD, TRACK, SPM, CAP>(a, X, L, k0 + kk, lane, ring_in, ring_out, selr, tmax, row1, bs, bi,
                                                bj, sp_ptr, smask);
        return tmax;
    }

    // The hot path: no guard, no tracking; SP1 = this warp holds special rows
    // that are strip-bottom rows (k a multiple of ALPHA): predicated stores.
    template <bool SP1>
    static __device__ __forceinline__ int tile_fast(const FillArgs &a, const StepInfo &X, Lane &L, int c, int lane,
                                                    uint32_t ring_in, uint32_t ring_out, uint32_t selr,
                                                    int *sp_ptr)
    {
        int tmax = INT_MIN;
        int d0 = 0, d1 = 0, d2 = 0;
        const int k0 = c * STEPS;
#pragma unroll 2
        for (int kk = 0; kk < STEPS; kk++)
            tmax = step<false, false, SP1 ? 1 : 0>(a, X, L, k0 + kk, lane, ring_in, ring_out, selr, tmax, 0, d0, d1,
                                                   d2, sp_ptr, 0u);
        return tmax;
    }

    static __device__ __forceinline__ void save(const Lane &L, int *sv, int lane)
    {
#pragma unroll
        for (int r = 0; r < ALPHA; r++) {
            sv[r * 32 + lane] = L.e[r];
            sv[(ALPHA + r) * 32 + lane] = L.t[r];
        }
        sv[(2 * ALPHA) * 32 + lane] = L.tprev;
        sv[(2 * ALPHA + 1) * 32 + lane] = L.out_t0;
        sv[(2 * ALPHA + 2) * 32 + lane] = L.out_f0;
        sv[(2 * ALPHA + 3) * 32 + lane] = L.out_t1;
        sv[(2 * ALPHA + 4) * 32 + lane] = L.out_f1;
    }
    static __device__ __forceinline__ void restore(Lane &L, const int *sv, int lane)
    {
#pragma unroll
        for (int r = 0; r < ALPHA; r++) {
            L.e[r] = sv[r * 32 + lane];
            L.t[r] = sv[(ALPHA + r) * 32 + lane];
        }
        L.tprev = sv[(2 * ALPHA) * 32 + lane];
        L.out_t0 = sv[(2 * ALPHA + 1) * 32 + lane];
        L.out_f0 = sv[(2 * ALPHA + 2) * 32 + lane];
        L.out_t1 = sv[(2 * ALPHA + 3) * 32 + lane];
        L.out_f1 = sv[(2 * ALPHA + 4) * 32 + lane];
    }
};

// Boundary values of row 0 / column 0 as t = H - G_first (reading S3, and the
// global initialisation of reading S9): column index j is the GLOBAL 0-based
// column (DP column j+1).
template <bool LOCAL>
__device__ __forceinline__ int2 top_boundary(const FillArgs &a, int j)
{
    if (LOCAL) return make_int2(-a.gf, NEG);
    return make_int2(-(a.go + (j + 1) * a.ge) - a.gf, NEG);  // H(0, j+1) = -(G_open + (j+1) G_ext)
}

__device__ __forceinline__ int ld_acquire_sys(const int *p)
{
    int v;
    asm volatile("ld.acquire.sys.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys_s32(int *p, int v)
{
    asm volatile("st.release.sys.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ int2 ld_sys_int2(const int2 *p)
{
    int2 v;
    asm volatile("ld.relaxed.sys.global.v2.s32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p) : "memory");
    return v;
}

template <int ALPHA, int NW, int W, bool LOCAL, bool WIDE = false>
__global__ void __launch_bounds__((NW + 1) * 32) sw_fill_kernel(const __grid_constant__ FillArgs a)
{
    using F = Fill<ALPHA, NW, W, LOCAL, WIDE>;
    constexpr int RING = F::RING, SRING = F::SRING, BH = F::BH, SKEW = F::SKEW, STEPS = F::STEPS, LAG = F::LAG;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int2 *rings = reinterpret_cast<int2 *>(smem_raw);                        // (NW+1) x RING
    uint32_t *selr = reinterpret_cast<uint32_t *>(rings + (NW + 1) * RING);  // SRING
    int *saves = reinterpret_cast<int *>(selr + SRING);                     // NW x NSAVE x 32
    __shared__ int s_band, s_abort;

    const int warp = threadIdx.x >> 5, lane = lane_id();
    const uint32_t selr_base = (uint32_t)__cvta_generic_to_shared(selr);
    const StripeArgs &S = a.st[blockIdx.x % a.nstripes];
    const int NT = S.NT;
    const bool has_left = S.lb != nullptr, has_right = S.rb != nullptr;
    int bs = 0, bi = LOCAL ? 0 : INT_MAX, bj = LOCAL ? 0 : INT_MAX;
    long long nrep = 0;
    if (*a.err) return;
    StepInfo X;
    X.w = S.w;
    X.col0 = S.col0;
    X.sp_ld = S.sp_ld;
    X.sp_stride = S.sp_stride;
    X.jcap = S.w - 1;
    X.rbrow = nullptr;
    X.hw = LOCAL ? S.w : min(S.w, a.hit_w);
    // tiles in which a lane meets the capture column jcap (lane l at step jcap/2 + l)
    const int cap_t0 = (X.jcap >> 1) / STEPS, cap_t1 = ((X.jcap >> 1) + 31) / STEPS;

    X.sp_end = S.sp != nullptr ? S.sp + (long long)a.sp_slots * S.sp_stride : nullptr;
    X.sp_span = (long long)a.sp_slots * S.sp_stride;
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
        const int G = a.band_base + b;         // global band number (progress, colp)
        const int rowtop = a.row_base + b * BH;  // 0-based first row of the band
        if (a.dbg && threadIdx.x == 0 && S.col0 == 0) a.dbg[80 * G] = gtimer();

        typename F::Lane L;
        const int row0 = rowtop + (warp * 32 + lane) * ALPHA;  // 0-based first row of the strip
        int *sp_ptr = nullptr;
        uint32_t smask = 0;
        bool warp_sp = false;
        X.rbrow = S.rb != nullptr ? S.rb + row0 + 1 : nullptr;
        if (warp < NW) {
            const uint32_t w = row0 < a.m ? a.A2[row0 >> 4] : 0u;
            const int sh = (row0 & 15) * 2;
#pragma unroll
            for (int r = 0; r < ALPHA; r++) {
                const uint32_t code = (w >> (sh + 2 * r)) & 3u;
                L.P[r] = (row0 + r < a.m) ? (WIDE ? code : a.prof[code]) : (WIDE ? 5u : PADPROF);
                L.e[r] = NEG;
                // H(i,0) - G_first; -inf when the anchor is a gap crosspoint (S20)
                L.t[r] = LOCAL ? -a.gf : a.anchor_gap ? NEG : -(a.go + (row0 + r + 1) * a.ge) - a.gf;
            }
            L.tprev = LOCAL ? -a.gf : a.anchor_gap ? NEG : (row0 == 0 ? -a.gf : -(a.go + row0 * a.ge) - a.gf);
            L.out_t0 = L.out_f0 = L.out_t1 = L.out_f1 = 0;
            if (LOCAL && a.k > 0) {
                // special rows among DP rows row0+1 .. row0+ALPHA (<= m); the band's
                // bottom row is written by the I/O warp from its coalesced drain
                const int bottom = rowtop + BH;
                for (int r = 0; r < ALPHA; r++) {
                    const int row = row0 + r + 1;
                    if (row <= a.m && row % a.k == 0 && row != bottom) smask |= 1u << r;
                }
                if (smask) {
                    const int first = __ffs(smask) - 1;
                    sp_ptr = sp_row(a, S, (row0 + first + 1) / a.k - 1);
                }
            }
            warp_sp = __any_sync(0xffffffffu, smask != 0);
        }
        const int spm = (a.k > 0 && a.k % ALPHA == 0) ? 1 : 2;

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
                }
                __syncwarp();
            }
            int2 *ring0 = rings;
#pragma unroll
            for (int x = lane; x < W; x += 32) {
                const int col = c * W + x;
                int2 v = (rowtop == 0) ? top_boundary<LOCAL>(a, S.col0 + col) : __ldcg(S.rowb_in + col);
                ring0[col & (RING - 1)] = v;
                uint32_t code = 4u;
                if (col < S.w) {
                    const int gc = S.col0 + col;
                    code = (__ldg(a.B2 + (gc >> 4)) >> ((gc & 15) * 2)) & 3u;
                }
                selr[col & (SRING - 1)] = WIDE ? (code == 4u ? 6u : code) : col_sel(code);
            }
        };
        // special row that is this band's bottom row: written here, coalesced
        int *io_sp = nullptr;
        if (LOCAL && a.k > 0) {
            const int bottom = rowtop + BH;
            if (bottom <= a.m && bottom % a.k == 0) io_sp = sp_row(a, S, bottom / a.k - 1);
        }
        unsigned int *const colp = (LOCAL && band_has_special(rowtop, BH, a.m, a.k)) ? S.colp : nullptr;
        auto io_drain = [&](int cd) {
            const int2 *ringN = rings + NW * RING;
#pragma unroll
            for (int x = lane; x < W; x += 32) {
                const int col = cd * W - SKEW + x;
                if (col >= 0) {
                    const int2 v = ringN[col & (RING - 1)];
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
        // left border of this warp's rows (stripes after the first): wait for the
        // left neighbour's flags, then take (t, E) at column col0 - 1 as the state.
        auto load_left = [&]() {
            if (lane == 0) {
                const int fi = b * NW + warp;
                const unsigned long long t0 = gtimer();
                while (ld_acquire_sys(S.lready + fi) != a.epoch || (fi > 0 && ld_acquire_sys(S.lready + fi - 1) != a.epoch)) {
                    if (gtimer() - t0 > (unsigned long long)a.timeout_ns) { atomicExch(a.err, 2); break; }
                    __nanosleep(64);
                }
            }
            __syncwarp();
#pragma unroll
            for (int r = 0; r < ALPHA; r++) {
                const int2 v = ld_sys_int2(S.lb + row0 + 1 + r);  // rows past m read padding, never used
                L.t[r] = v.x;
                L.e[r] = v.y;
            }
            if (row0 > 0) L.tprev = ld_sys_int2(S.lb + row0).x;
            else L.tprev = LOCAL ? -a.gf : -(a.go + S.col0 * a.ge) - a.gf;  // t(0, col0 - 1)
        };

        if (warp == NW) io_load(0);
        __syncthreads();
        if (a.dbg && threadIdx.x == 0 && S.col0 == 0) a.dbg[80 * G + 1] = gtimer();
        const int S_END = NT + LAG * (NW - 1);
        int *sv = saves + warp * F::NSAVE * 32;
        for (int s = 0; s <= S_END; ++s) {
            if (a.dbg && threadIdx.x == 0 && S.col0 == 0 && (s == NT / 4 || s == NT / 2 || s == 3 * NT / 4))
                a.dbg[80 * G + 2 + (s == NT / 2) + 2 * (s == 3 * NT / 4)] = gtimer();
            if (warp < NW) {
                const int c = s - LAG * warp;
                if (c >= 0 && c < NT) {
                    const uint32_t rin = pin((uint32_t)__cvta_generic_to_shared(rings + warp * RING));
                    const uint32_t rout = pin((uint32_t)__cvta_generic_to_shared(rings + (warp + 1) * RING));
                    const uint32_t selr_s = pin(selr_base);
                    if (c == 0 && has_left) load_left();
                    int thr;
                    // loaded here, used after the tile (the L2 round trip overlaps it)
                    const int gbest = LOCAL ? ld_relaxed(a.gbest) : 0;
                    const int bs0 = bs;
                    F::save(L, sv, lane);
                    int tmax;
                    const bool cap = has_right && c >= cap_t0 && c <= cap_t1;
                    if (cap) {
                        tmax = F::template tile<true, false, 2, true>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, smask);
                        if (c == cap_t1) {
                            // this warp's rows are complete at the stripe's last column
                            __threadfence_system();
                            __syncwarp();
                            if (lane == 0 && S.rready != nullptr) st_release_sys_s32(S.rready + b * NW + warp, a.epoch);
                        }
                    } else if (c < F::GUARD_TILES || (warp_sp && spm == 2)) {
                        tmax = F::template tile<true, false, 2>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, sp_ptr, smask);
                    } else if (warp_sp) {
                        tmax = F::template tile_fast<true>(a, X, L, c, lane, rin, rout, selr_s, sp_ptr);
                    } else {
                        tmax = F::template tile_fast<false>(a, X, L, c, lane, rin, rout, selr_s, nullptr);
                    }
                    thr = LOCAL ? max(max(bs0, gbest), 1) : a.goal;
                    if (__any_sync(0xffffffffu, tmax >= thr - a.gf)) {  // tmax is over t = H - G_first
                        // exact replay of this tile from the saved state (rare)
                        F::restore(L, sv, lane);
                        const int obs = bs, obi = bi, obj = bj;
                        F::template tile<true, true, 0>(a, X, L, c, lane, rin, rout, selr_s, row0 + 1, bs, bi, bj, nullptr, 0u);
                        if (lane == 0) nrep++;
                        if (LOCAL) {
                            if (bs > obs) atomicMax(a.gbest, bs);
                        } else if (bi != obi || bj != obj) {
                            atomicMin(a.hit_key, ((unsigned long long)(unsigned)bi << 32) | (unsigned)bj);
                            atomicMin(a.hit_band, b);
                        }
                    }
                }
            } else {
                if (s + 1 < NT) io_load(s + 1);
                const int cd = s - 1 - LAG * (NW - 1);
                if (cd >= 0) io_drain(cd);
                if (!LOCAL && lane == 0 && ld_relaxed(a.hit_band) < b) s_abort = 1;
            }
            __syncthreads();
            if (s_abort) break;
        }
        if (warp == NW && lane == 0 && !s_abort) publish_progress(a, S, G, INT_MAX);
        if (!LOCAL && a.match && !s_abort) {
            // Stage-2 goal-based matching: the
            // capture tiles left (t, E) of the special row's DP column for
            // every row of the band in S.rb; row j' is original column
            // j = j_c - j', t + G_first the reverse H there, E the reverse F.
            // Coalesced, once per band (per-lane matching inside the capture
            // tiles stalled each warp on dependent global loads).
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
                // after every start hit of the same row (DP columns <= w - 1): the sweep order S19
                if (kind >= 0) key = min(key, ((unsigned long long)(unsigned)row << 32) | (unsigned)(S.w + kind));
            }
            if (key != ~0ull) {
                atomicMin(a.hit_key, key);
                atomicMin(a.hit_band, b);
            }
        }
        if (a.dbg && threadIdx.x == 0 && S.col0 == 0) a.dbg[80 * G + 15] = gtimer();
        if (LOCAL && a.k > 0) {
            // publish this band's special rows (this stripe's slice) to the host
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

    // ---------------------------------------------------------------- final per-CTA reduction
    if (lane == 0 && nrep) atomicAdd(a.replays, (unsigned long long)nrep);
    if (LOCAL) {
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
