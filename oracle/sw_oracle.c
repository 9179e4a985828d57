/*
 * oracle/sw_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct, single-threaded CPU implementation of
 * the computation CUDAlign 2.0's Stage 1 performs (Sandes & de Melo,
 * IPDPS 2011; /root/reference/PAPER.md, cited below as P:<line>).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path
 * (paper_conf_ipps_sandesm11_b200/) never includes, links or calls it, and
 * this file includes nothing from the product path.
 *
 * Notation follows the paper: S0 (length m, rows i) and S1 (length n,
 * columns j); matrices H, E, F (Eq. 1-3); ma, mi
 * the match / mismatch scores; G_first the first-gap penalty,
 * G_ext the extension penalty, G_open = G_first - G_ext.
 *
 * Readings of the paper that this file takes:
 *   S1  Eq. 1 is read as H_{i-1,j-1} + p(i,j) with a signed p (P:62-64,
 *       P:315, Table X).
 *   S2  the API's gap_open is G_open, so G_first = gap_open + gap_ext.
 *   S3  E(i,0) = F(0,j) = -infinity (NEG below); H(i,0) = H(0,j) = 0.
 *   S4  argmax tie-break: highest score, then smallest i, then smallest j;
 *       score 0 reports (0,0).  Implemented as a row-major scan with '>'.
 *   S5/S6 special rows hold columns 1..n of H and F for every i = k,2k,..<=m.
 *   S7  characters are compared case-insensitively (codes A,C,G,T).
 *   S9/S10 reverse pass: anchored global recurrence on the reversed
 *       prefixes; first hit in row-major order of the reverse matrix.
 *   S18-S22 Stage 2 (or_stage2): junction rules, anchor initialisation by
 *       crosspoint type, event order of the orthogonal sweep, termination.
 *
 * Arithmetic: int64 everywhere (wider than any kernel; the paper uses
 * 4-byte cells, and all values here stay far inside int32).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define NEG (-(int64_t)1 << 40) /* "minus infinity": never produced by a real cell */

typedef struct {
    int64_t score;
    int64_t i;
    int64_t j;
} or_result;

typedef int (*or_row_sink)(void *user, int64_t row, const int64_t *H, const int64_t *F, int64_t n);

static int up(char c) { return (c >= 'a' && c <= 'z') ? c - 32 : c; }

/* p(i,j) = ma if S0[i] = S1[j] (match) and mi otherwise. */
static int64_t p_score(char a, char b, int64_t ma, int64_t mi) { return up(a) == up(b) ? ma : mi; }

static int64_t max2(int64_t a, int64_t b) { return a > b ? a : b; }

/*
 * Stage 1, linear space: row-by-row fill of Eq. 1-3 keeping
 * one previous row of H and F; E is carried along the row.  Returns the
 * best score and the first (row-major) cell holding it.
 * Every k-th row (k > 0) is handed to `sink` as H[1..n], F[1..n].
 */
int or_stage1(const char *S0, int64_t m, const char *S1, int64_t n, int64_t ma, int64_t mi,
              int64_t G_open, int64_t G_ext, int64_t k, or_row_sink sink, void *user,
              or_result *best)
{
    const int64_t G_first = G_open + G_ext;
    int64_t *Hprev = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Fprev = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Hcur = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Fcur = malloc((size_t)(n + 1) * sizeof(int64_t));
    if (!Hprev || !Fprev || !Hcur || !Fcur) {
        free(Hprev); free(Fprev); free(Hcur); free(Fcur);
        return -1;
    }
    /* "the first row and column are filled with zeroes" */
    for (int64_t j = 0; j <= n; j++) { Hprev[j] = 0; Fprev[j] = NEG; }
    best->score = 0; best->i = 0; best->j = 0;
    for (int64_t i = 1; i <= m; i++) {
        int64_t E = NEG; /* E(i,0) */
        Hcur[0] = 0;
        Fcur[0] = NEG;
        for (int64_t j = 1; j <= n; j++) {
            /* Eq. 2: E_{i,j} = max(E_{i,j-1} - G_ext, H_{i,j-1} - G_first) */
            E = max2(E - G_ext, Hcur[j - 1] - G_first);
            /* Eq. 3: F_{i,j} = max(F_{i-1,j} - G_ext, H_{i-1,j} - G_first) */
            Fcur[j] = max2(Fprev[j] - G_ext, Hprev[j] - G_first);
            /* Eq. 1: H_{i,j} = max(0, E_{i,j}, F_{i,j}, H_{i-1,j-1} + p(i,j)) */
            int64_t h = 0;
            h = max2(h, E);
            h = max2(h, Fcur[j]);
            h = max2(h, Hprev[j - 1] + p_score(S0[i - 1], S1[j - 1], ma, mi));
            Hcur[j] = h;
            if (h > best->score) { best->score = h; best->i = i; best->j = j; }
        }
        if (k > 0 && i % k == 0 && sink) {
            if (sink(user, i, Hcur + 1, Fcur + 1, n)) {
                free(Hprev); free(Fprev); free(Hcur); free(Fcur);
                return -2;
            }
        }
        int64_t *t;
        t = Hprev; Hprev = Hcur; Hcur = t;
        t = Fprev; Fprev = Fcur; Fcur = t;
    }
    free(Hprev); free(Fprev); free(Hcur); free(Fcur);
    return 0;
}

/*
 * The same definition with the whole (m+1) x (n+1) matrices kept, for
 * tiny inputs: H, E, F are row-major with row stride n+1.  Boundary cells
 * hold H = 0, E = F = NEG (reading S3).
 */
int or_full_matrix(const char *S0, int64_t m, const char *S1, int64_t n, int64_t ma, int64_t mi,
                   int64_t G_open, int64_t G_ext, int64_t *H, int64_t *E, int64_t *F)
{
    const int64_t G_first = G_open + G_ext;
    const int64_t w = n + 1;
    for (int64_t i = 0; i <= m; i++)
        for (int64_t j = 0; j <= n; j++) {
            if (i == 0 || j == 0) {
                H[i * w + j] = 0;
                E[i * w + j] = NEG;
                F[i * w + j] = NEG;
                continue;
            }
            E[i * w + j] = max2(E[i * w + j - 1] - G_ext, H[i * w + j - 1] - G_first);     /* Eq. 2 */
            F[i * w + j] = max2(F[(i - 1) * w + j] - G_ext, H[(i - 1) * w + j] - G_first); /* Eq. 3 */
            int64_t h = 0;                                                                   /* Eq. 1 */
            h = max2(h, E[i * w + j]);
            h = max2(h, F[i * w + j]);
            h = max2(h, H[(i - 1) * w + j - 1] + p_score(S0[i - 1], S1[j - 1], ma, mi));
            H[i * w + j] = h;
        }
    return 0;
}

/*
 * One band of Stage 1: given row r0's H[0..n], F[0..n] (column 0 included:
 * H = 0, F = NEG), compute rows r0+1..r1 and return row r1 in Hbot/Fbot
 * (length n+1) plus the band's best (score, i, j) under the same order.
 * Used to check special rows produced at scale by induction: row r0 + k
 * must equal band(row r0).
 */
int or_band(const char *S0, int64_t m, const char *S1, int64_t n, int64_t ma, int64_t mi,
            int64_t G_open, int64_t G_ext, int64_t r0, int64_t r1, const int64_t *Htop,
            const int64_t *Ftop, int64_t *Hbot, int64_t *Fbot, or_result *best)
{
    const int64_t G_first = G_open + G_ext;
    if (r0 < 0 || r1 < r0 || r1 > m) return -1;
    int64_t *Hprev = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Fprev = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Hcur = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Fcur = malloc((size_t)(n + 1) * sizeof(int64_t));
    if (!Hprev || !Fprev || !Hcur || !Fcur) {
        free(Hprev); free(Fprev); free(Hcur); free(Fcur);
        return -1;
    }
    memcpy(Hprev, Htop, (size_t)(n + 1) * sizeof(int64_t));
    memcpy(Fprev, Ftop, (size_t)(n + 1) * sizeof(int64_t));
    best->score = 0; best->i = 0; best->j = 0;
    for (int64_t i = r0 + 1; i <= r1; i++) {
        int64_t E = NEG;
        Hcur[0] = 0;
        Fcur[0] = NEG;
        for (int64_t j = 1; j <= n; j++) {
            E = max2(E - G_ext, Hcur[j - 1] - G_first);
            Fcur[j] = max2(Fprev[j] - G_ext, Hprev[j] - G_first);
            int64_t h = 0;
            h = max2(h, E);
            h = max2(h, Fcur[j]);
            h = max2(h, Hprev[j - 1] + p_score(S0[i - 1], S1[j - 1], ma, mi));
            Hcur[j] = h;
            if (h > best->score) { best->score = h; best->i = i; best->j = j; }
        }
        int64_t *t;
        t = Hprev; Hprev = Hcur; Hcur = t;
        t = Fprev; Fprev = Fcur; Fcur = t;
    }
    memcpy(Hbot, Hprev, (size_t)(n + 1) * sizeof(int64_t));
    memcpy(Fbot, Fprev, (size_t)(n + 1) * sizeof(int64_t));
    free(Hprev); free(Fprev); free(Hcur); free(Fcur);
    return 0;
}

/*
 * Global (Needleman-Wunsch style) Gotoh score of S0[1..m] vs S1[1..n]:
 * the recurrence of Eq. 1-3 without the 0 term, with the textbook global
 * initialisation H(0,0) = 0, H(0,j) = E(0,j) = -(G_open + j G_ext),
 * H(i,0) = F(i,0) = -(G_open + i G_ext), E(i,0) = F(0,j) = -infinity.
 * This is the "global recurrence" Stage 2 runs (reading S9).
 */
int64_t or_global(const char *S0, int64_t m, const char *S1, int64_t n, int64_t ma, int64_t mi,
                  int64_t G_open, int64_t G_ext)
{
    const int64_t G_first = G_open + G_ext;
    int64_t *Hprev = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Fprev = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Hcur = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Fcur = malloc((size_t)(n + 1) * sizeof(int64_t));
    Hprev[0] = 0;
    Fprev[0] = NEG;
    for (int64_t j = 1; j <= n; j++) { Hprev[j] = -(G_open + j * G_ext); Fprev[j] = NEG; }
    for (int64_t i = 1; i <= m; i++) {
        Hcur[0] = -(G_open + i * G_ext);
        Fcur[0] = Hcur[0];
        int64_t E = NEG;
        for (int64_t j = 1; j <= n; j++) {
            E = max2(E - G_ext, Hcur[j - 1] - G_first);
            Fcur[j] = max2(Fprev[j] - G_ext, Hprev[j] - G_first);
            int64_t h = max2(E, Fcur[j]);
            h = max2(h, Hprev[j - 1] + p_score(S0[i - 1], S1[j - 1], ma, mi));
            Hcur[j] = h;
        }
        int64_t *t;
        t = Hprev; Hprev = Hcur; Hcur = t;
        t = Fprev; Fprev = Fcur; Fcur = t;
    }
    int64_t r = (m == 0 && n == 0) ? 0 : Hprev[n];
    if (m == 0 && n > 0) r = -(G_open + n * G_ext);
    free(Hprev); free(Fprev); free(Hcur); free(Fcur);
    return r;
}

/*
 * Reverse pass (Stage 2 reuse of the Stage-1 engine):
 * reverse the prefixes S0[1..i_end] and S1[1..j_end], run the global
 * recurrence (or_global's initialisation, no 0 term) and return the first
 * cell (i', j'), i', j' >= 1, in row-major order of the reverse matrix with
 * H = goal.  The forward start is (i_end - i', j_end - j'): the DP cell
 * *before* the first aligned pair (reading S8, Table III).
 * goal == 0 returns the end itself.  Returns 1 if found, 0 if not.
 */
int or_reverse_goal(const char *S0, int64_t i_end, const char *S1, int64_t j_end, int64_t ma,
                    int64_t mi, int64_t G_open, int64_t G_ext, int64_t goal, or_result *start)
{
    const int64_t G_first = G_open + G_ext;
    if (goal == 0) { start->score = 0; start->i = i_end; start->j = j_end; return 1; }
    const int64_t m = i_end, n = j_end;
    char *R0 = malloc((size_t)m + 1), *R1 = malloc((size_t)n + 1);
    for (int64_t i = 0; i < m; i++) R0[i] = S0[i_end - 1 - i];
    for (int64_t j = 0; j < n; j++) R1[j] = S1[j_end - 1 - j];
    int64_t *Hprev = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Fprev = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Hcur = malloc((size_t)(n + 1) * sizeof(int64_t));
    int64_t *Fcur = malloc((size_t)(n + 1) * sizeof(int64_t));
    Hprev[0] = 0;
    Fprev[0] = NEG;
    for (int64_t j = 1; j <= n; j++) { Hprev[j] = -(G_open + j * G_ext); Fprev[j] = NEG; }
    int found = 0;
    for (int64_t i = 1; i <= m && !found; i++) {
        Hcur[0] = -(G_open + i * G_ext);
        Fcur[0] = Hcur[0];
        int64_t E = NEG;
        for (int64_t j = 1; j <= n; j++) {
            E = max2(E - G_ext, Hcur[j - 1] - G_first);
            Fcur[j] = max2(Fprev[j] - G_ext, Hprev[j] - G_first);
            int64_t h = max2(E, Fcur[j]);
            h = max2(h, Hprev[j - 1] + p_score(R0[i - 1], R1[j - 1], ma, mi));
            Hcur[j] = h;
            if (!found && h == goal) {
                found = 1;
                start->score = goal;
                start->i = i_end - i;
                start->j = j_end - j;
            }
        }
        int64_t *t;
        t = Hprev; Hprev = Hcur; Hcur = t;
        t = Fprev; Fprev = Fcur; Fcur = t;
    }
    free(R0); free(R1); free(Hprev); free(Fprev); free(Hcur); free(Fcur);
    return found;
}

/*
 * Flush-interval rule: the flush interval, in blocks of alpha*T
 * rows, must be at least ceil(8 m n / (alpha T |SRA|)).  Returns the
 * special-row spacing R = alpha*T * ceil(8 m n / (alpha T |SRA|)) in rows.
 */
int64_t or_flush_rows(int64_t m, int64_t n, int64_t alphaT, int64_t sra_bytes)
{
    /* 8 m n can exceed 2^63 for huge inputs: compute with long double and fix up. */
    long double num = 8.0L * (long double)m * (long double)n;
    long double den = (long double)alphaT * (long double)sra_bytes;
    int64_t q = (int64_t)(num / den);
    while ((long double)q * den < num) q++;
    while (q > 0 && (long double)(q - 1) * den >= num) q--;
    if (q < 1) q = 1;
    return alphaT * q;
}

/*
 * Stage 2, partial traceback, plainly: from the end point
 * C = (i_end, j_end, best, 0) back to the start point, one partition at a
 * time, returning the crosspoint list L_2 in ascending order
 * (start point first, end point last).  A crosspoint is (i, j, score, type),
 * type 0 = match/mismatch, 2 = gap in S1 (a vertical gap, matrix F).
 *
 * One iteration, for the current crosspoint (i_c, j_c, g, type):
 *  - the partition is rows r..i_c, r = the nearest special row strictly above
 *    i_c (r = ((i_c - 1) / k) k; r = 0 means "none": row 0 then plays the
 *    special row with H = 0, F = -infinity, the local boundary, reading S21);
 *  - the reverse DP is the global recurrence anchored at (i_c, j_c)
 *    over i' = i_c - i in [0, i_c - r], j' = j_c - j in [0, j_c]:
 *    H'(0,0) = 0, column j' = 0: H' = F' = -(G_open + i' G_ext), E' = -inf;
 *    row i' = 0: H' = E' = -(G_open + j' G_ext), F' = -inf.  When the anchor
 *    is a gap crosspoint (type 2) the path must leave it by continuing that
 *    vertical gap, so the row i' = 0 (j' >= 1) is -infinity and so is the
 *    diagonal out of the anchor ("the initialization must be adjusted not to
 *    consider a duplicated gap open penalty"; reading S20);
 *  - events, in the order of the orthogonal sweep (Fig. 7: vertical
 *    strips j' = 0, 1, 2, ...; reading S19), the first one wins:
 *      start:   H'(i', j') == g for 1 <= i' < i_c - r  -> the start point
 *               (i_c - i', j_c - j', 0, 0);
 *      H-match: Hs(j) + H'(i_c - r, j') == g           -> (r, j, Hs(j), 0);
 *      F-match: Fs(j) + F'(i_c - r, j') + G_open == g  -> (r, j, Fs(j), 2)
 *               (a vertical gap crossing row r is charged G_open once, not
 *               twice; reading S18), where j = j_c - j' and Hs, Fs are
 *               the special row r of Stage 1 (Hs(0) = 0, Fs(0) = -inf);
 *      within one strip: starts by increasing i', then H-match, then F-match.
 *  - the new crosspoint's score is the special row's H, or its F for a gap
 *    (P:233); the loop ends at a crosspoint with score 0 and type 0 (the
 *    start point; a gap crosspoint may have a score <= 0, reading S22).
 * The special rows are recomputed here with or_stage1 (rows k, 2k, ...).
 * Returns the number of crosspoints (writes min(count, cap) of them), or
 * -1 (allocation), -3 (no event: inconsistent inputs).
 */
typedef struct {
    int64_t i;
    int64_t j;
    int64_t score;
    int64_t type;
} or_crosspoint;

typedef struct {
    int64_t n, k, count;
    int64_t *H, *F; /* count rows of n + 1 values (column 0 included) */
} or_rows;

static int keep_row(void *user, int64_t row, const int64_t *H, const int64_t *F, int64_t n)
{
    or_rows *R = (or_rows *)user;
    int64_t q = row / R->k - 1;
    R->H[q * (n + 1)] = 0;   /* H(r, 0) = 0   (local boundary, reading S3) */
    R->F[q * (n + 1)] = NEG; /* F(r, 0) = -inf */
    memcpy(R->H + q * (n + 1) + 1, H, (size_t)n * sizeof(int64_t));
    memcpy(R->F + q * (n + 1) + 1, F, (size_t)n * sizeof(int64_t));
    R->count = q + 1;
    return 0;
}

int64_t or_stage2(const char *S0, int64_t m, const char *S1, int64_t n, int64_t ma, int64_t mi,
                  int64_t G_open, int64_t G_ext, int64_t k, int64_t best, int64_t i_end, int64_t j_end,
                  or_crosspoint *out, int64_t cap)
{
    const int64_t G_first = G_open + G_ext;
    or_rows R = {n, k, 0, NULL, NULL};
    const int64_t nrows = k > 0 ? m / k : 0;
    if (nrows > 0) {
        R.H = malloc((size_t)(nrows * (n + 1)) * sizeof(int64_t));
        R.F = malloc((size_t)(nrows * (n + 1)) * sizeof(int64_t));
        if (!R.H || !R.F) { free(R.H); free(R.F); return -1; }
        or_result b1;
        or_stage1(S0, m, S1, n, ma, mi, G_open, G_ext, k, keep_row, &R, &b1);
    }
    /* the list is built from the end point backwards */
    int64_t ncp = 0, capl = 16;
    or_crosspoint *L = malloc((size_t)capl * sizeof(or_crosspoint));
    or_crosspoint C = {i_end, j_end, best, 0};
    L[ncp++] = C;
    int64_t rc = 0;
    while (!(C.score == 0 && C.type == 0)) {
        const int64_t ic = C.i, jc = C.j, g = C.score;
        const int64_t r = k > 0 ? ((ic - 1) / k) * k : 0;
        const int64_t Lr = ic - r;
        const int64_t w = jc + 1;
        int64_t *RH = malloc((size_t)((Lr + 1) * w) * sizeof(int64_t));
        int64_t *RE = malloc((size_t)((Lr + 1) * w) * sizeof(int64_t));
        int64_t *RF = malloc((size_t)((Lr + 1) * w) * sizeof(int64_t));
        if (!RH || !RE || !RF) { free(RH); free(RE); free(RF); rc = -1; break; }
        for (int64_t a = 0; a <= Lr; a++)
            for (int64_t b = 0; b <= jc; b++) {
                int64_t *h = &RH[a * w + b], *e = &RE[a * w + b], *f = &RF[a * w + b];
                if (a == 0 && b == 0) { *h = 0; *e = NEG; *f = NEG; continue; }
                if (b == 0) { *h = -(G_open + a * G_ext); *f = *h; *e = NEG; continue; }
                if (a == 0) {
                    if (C.type == 2) { *h = NEG; *e = NEG; }
                    else { *h = -(G_open + b * G_ext); *e = *h; }
                    *f = NEG;
                    continue;
                }
                *e = max2(RE[a * w + b - 1] - G_ext, RH[a * w + b - 1] - G_first); /* Eq. 2 */
                *f = max2(RF[(a - 1) * w + b] - G_ext, RH[(a - 1) * w + b] - G_first); /* Eq. 3 */
                int64_t diag = RH[(a - 1) * w + b - 1];
                if (a == 1 && b == 1 && C.type == 2) diag = NEG;
                /* reversed sequences: row i' pairs S0[ic - i' + 1] (1-based) */
                *h = max2(max2(*e, *f), diag + p_score(S0[ic - a], S1[jc - b], ma, mi)); /* Eq. 1, no 0 */
            }
        const int64_t *Hs = r > 0 ? R.H + (r / k - 1) * (n + 1) : NULL;
        const int64_t *Fs = r > 0 ? R.F + (r / k - 1) * (n + 1) : NULL;
        int found = 0;
        or_crosspoint X = {0, 0, 0, 0};
        for (int64_t b = 0; b <= jc && !found; b++) {
            for (int64_t a = 1; a < Lr && !found; a++)
                if (RH[a * w + b] == g) { X.i = ic - a; X.j = jc - b; X.score = 0; X.type = 0; found = 1; }
            if (found) break;
            const int64_t j = jc - b;
            const int64_t hs = Hs ? Hs[j] : 0, fs = Fs ? Fs[j] : NEG;
            if (hs + RH[Lr * w + b] == g) { X.i = r; X.j = j; X.score = hs; X.type = 0; found = 1; break; }
            if (fs > NEG / 2 && RF[Lr * w + b] > NEG / 2 && fs + RF[Lr * w + b] + G_open == g) {
                X.i = r; X.j = j; X.score = fs; X.type = 2; found = 1; break;
            }
        }
        free(RH); free(RE); free(RF);
        if (!found) { rc = -3; break; }
        if (ncp == capl) { capl *= 2; L = realloc(L, (size_t)capl * sizeof(or_crosspoint)); }
        L[ncp++] = X;
        C = X;
    }
    if (rc == 0) {
        for (int64_t q = 0; q < ncp && q < cap; q++) out[q] = L[ncp - 1 - q];
        rc = ncp;
    }
    free(L); free(R.H); free(R.F);
    return rc;
}

/*
 * Stages 3-5 for one partition P = (C_s, C_e) of L_k:
 * the optimal alignment of S0[i_s+1..i_e] with S1[j_s+1..j_e] that starts in
 * the state of C_s and ends in the state of C_e, by a full (h+1) x (w+1)
 * Gotoh matrix and its traceback (the definition the paper's Myers-Miller
 * stages reach in linear space; reading S23 in DESIGN.md):
 *
 *   types: 0 = match/mismatch (any state), 1 = gap in S0 (horizontal,
 *   matrix E), 2 = gap in S1 (vertical, matrix F);
 *   start: H(0,0) = 0, E(0,0) = 0 if type_s = 1 else -inf, F(0,0) = 0 if
 *   type_s = 2 else -inf -- a gap that crosses C_s continues at G_ext without
 *   a second opening;
 *   cells: Eq. 1-3 without the 0 term (global recurrence);
 *   end: the value of H, E or F at (h, w) by type_e.
 *
 * Writes the moves in forward order to ops ('M' diagonal pair, 'I' gap in S0
 * = horizontal, 'D' gap in S1 = vertical); returns the partition score, or
 * NEG if no alignment with these end states exists (-2 capacity / -1 memory
 * errors are reported through *nops = -1).  Traceback preference at equal
 * values: H state -> diagonal, then F, then E; E/F states -> extension, then
 * opening.
 */
int64_t or_align_partition(const char *S0, const char *S1, int64_t i_s, int64_t j_s, int64_t i_e, int64_t j_e,
                           int64_t ma, int64_t mi, int64_t G_open, int64_t G_ext, int64_t type_s,
                           int64_t type_e, char *ops, int64_t cap, int64_t *nops)
{
    const int64_t G_first = G_open + G_ext;
    const int64_t h = i_e - i_s, w = j_e - j_s, W = w + 1;
    *nops = -1;
    if (h < 0 || w < 0) return NEG;
    int64_t *H = malloc((size_t)((h + 1) * W) * sizeof(int64_t));
    int64_t *E = malloc((size_t)((h + 1) * W) * sizeof(int64_t));
    int64_t *F = malloc((size_t)((h + 1) * W) * sizeof(int64_t));
    if (!H || !E || !F) { free(H); free(E); free(F); return NEG; }
#define AT(M, a, b) M[(a) * W + (b)]
    for (int64_t a = 0; a <= h; a++)
        for (int64_t b = 0; b <= w; b++) {
            if (a == 0 && b == 0) {
                AT(H, 0, 0) = 0;
                AT(E, 0, 0) = type_s == 1 ? 0 : NEG;
                AT(F, 0, 0) = type_s == 2 ? 0 : NEG;
                continue;
            }
            const int64_t e = b > 0 ? max2(AT(E, a, b - 1) - G_ext, AT(H, a, b - 1) - G_first) : NEG; /* Eq. 2 */
            const int64_t f = a > 0 ? max2(AT(F, a - 1, b) - G_ext, AT(H, a - 1, b) - G_first) : NEG; /* Eq. 3 */
            const int64_t d = (a > 0 && b > 0) ? AT(H, a - 1, b - 1) + p_score(S0[i_s + a - 1], S1[j_s + b - 1], ma, mi)
                                               : NEG;                                                   /* Eq. 1 */
            AT(E, a, b) = e < NEG / 2 ? NEG : e;
            AT(F, a, b) = f < NEG / 2 ? NEG : f;
            const int64_t hv = max2(max2(e, f), d);
            AT(H, a, b) = hv < NEG / 2 ? NEG : hv;
        }
    const int64_t score = type_e == 1 ? AT(E, h, w) : type_e == 2 ? AT(F, h, w) : AT(H, h, w);
    if (score <= NEG / 2) { free(H); free(E); free(F); return NEG; }
    /* traceback from (h, w) in the end state */
    int64_t a = h, b = w, n = 0;
    int st = type_e == 1 ? 1 : type_e == 2 ? 2 : 0;
    char *rev = malloc((size_t)(h + w + 1));
    if (!rev) { free(H); free(E); free(F); return NEG; }
    while (a > 0 || b > 0) {
        if (st == 0) {
            if (a > 0 && b > 0 &&
                AT(H, a, b) == AT(H, a - 1, b - 1) + p_score(S0[i_s + a - 1], S1[j_s + b - 1], ma, mi)) {
                rev[n++] = 'M'; a--; b--;
            } else if (a > 0 && AT(H, a, b) == AT(F, a, b)) {
                st = 2;
            } else {
                st = 1;
            }
        } else if (st == 2) {
            rev[n++] = 'D';
            if (AT(F, a, b) == AT(F, a - 1, b) - G_ext && AT(F, a - 1, b) > NEG / 2) st = 2;
            else st = 0;
            a--;
        } else {
            rev[n++] = 'I';
            if (AT(E, a, b) == AT(E, a, b - 1) - G_ext && AT(E, a, b - 1) > NEG / 2) st = 1;
            else st = 0;
            b--;
        }
    }
#undef AT
    free(H); free(E); free(F);
    if (n > cap) { free(rev); return score; }
    for (int64_t q = 0; q < n; q++) ops[q] = rev[n - 1 - q];
    free(rev);
    *nops = n;
    return score;
}
