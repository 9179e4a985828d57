/*
 * cudalign_b200.h -- C ABI of the B200-native Stage-1 Smith-Waterman/Gotoh
 * engine (CUDAlign 2.0, Sandes & de Melo, IPDPS 2011; citations P:<line> are
 * lines of /root/reference/PAPER.md).
 *
 * What it computes:
 *   Stage 1: the Smith-Waterman matrix H with Gotoh affine gaps
 *   (Eq. 1-3) over S0 (m rows, i) and S1 (n columns, j) in linear
 *   space; the best score and its end cell; every k-th
 *   "special row" of H and F handed to the host.
 *   Reverse pass: the same engine on the reversed
 *   prefixes with the global recurrence, returning the start cell.
 *
 * Scoring convention (readings S1, S2 of DESIGN.md):
 *   match, mismatch : signed scores ADDED to H_{i-1,j-1} (Eq. 1 read as "+p").
 *   gap_open, gap_ext : non-negative penalties SUBTRACTED; a gap of length L
 *   costs gap_open + L*gap_ext, i.e. G_first = gap_open + gap_ext and
 *   G_ext = gap_ext.  The paper's experiments are (+1, -3, 3, 2)
 *   ("first gap -5, extension -2").
 *   Supported range: any scoring inside the SW_ERANGE rule.  Scorings with
 *   |match + gap_open + gap_ext| <= 127 and |mismatch + gap_open + gap_ext| <= 127
 *   use the int8 substitution profile (and the packed kernel when its value
 *   window allows); wider ones run the WIDE int32 kernels.
 *
 * Coordinates (reading S8): 1-based DP cells.  The end cell is the last
 * aligned pair; the start cell is the cell *before* the first aligned pair
 * (so end - start = length for a gapless alignment, Table III).
 *
 * Errors: every int-returning call returns SW_OK (0) or a negative code;
 * on error the output structs are left untouched.  There is no CPU fallback:
 * without a usable CUDA device sw_init fails with SW_ECUDA.
 *
 * Threading: one call at a time per context.  Special-row sinks are called
 * on the calling thread, in strictly ascending row order.
 */
#ifndef CUDALIGN_B200_H
#define CUDALIGN_B200_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SW_OK 0
#define SW_EINVAL (-1)     /* null pointer, negative size, bad scoring, bad device list */
#define SW_EALPHABET (-2)  /* a byte outside ACGTacgt (reading S7) */
#define SW_ERANGE (-3)     /* scores could leave the int32-safe range (+-2^30) */
#define SW_ENOMEM (-4)     /* device or pinned host allocation failed */
#define SW_ECUDA (-5)      /* CUDA runtime error (message via sw_last_error) */
#define SW_EABORTED (-6)   /* the special-row sink returned non-zero */
#define SW_ENOTFOUND (-7)  /* sw_reverse_goal: no cell equals goal (goal > H(i_end, j_end)) */

typedef struct sw_ctx sw_ctx;

/* Best (score, i, j).  Stage 1: highest score, then smallest i, then smallest
 * j (reading S4); (0, 0, 0) iff the best score is 0. */
typedef struct {
    int32_t score;
    int64_t i;
    int64_t j;
} sw_result;

/* Crosspoint: a cell (i, j) where the optimal alignment crosses a
 * special row, its score there and its type: 0 = match/mismatch (H), 2 = gap
 * in S1 (a vertical gap, matrix F).  The start point has score 0, type 0. */
typedef struct {
    int64_t i;
    int64_t j;
    int32_t score;
    int32_t type;
} sw_crosspoint;

/* Special-row sink: H and F are columns 1..n of DP row `row`, int32,
 * in library-owned pinned host memory valid only during the call.  Called
 * from the thread that called sw_align_stage1, rows strictly ascending.
 * A non-zero return aborts the alignment with SW_EABORTED. */
typedef int (*sw_row_sink)(void *user, int64_t row, const int32_t *H, const int32_t *F, int64_t n);

/* Timing breakdown of the last call (milliseconds, CUDA events on the
 * library's stream). */
typedef struct {
    double total_ms;   /* whole call (host API, includes copies) */
    double upload_ms;  /* host -> device copy of the sequences (0 for *_dev calls) */
    double encode_ms;  /* encode/pack kernel */
    double fill_ms;    /* the Stage-1 / reverse matrix-fill kernel */
    double reduce_ms;  /* best-cell reduction kernel + result copy */
    int64_t kernel_launches; /* kernels launched by the call */
    int64_t replays;   /* tiles replayed for exact argmax tracking */
    int64_t special_rows;
    int64_t special_bytes_d2h;
    int32_t alpha, warps, width, grid; /* launch configuration */
    int32_t patched;   /* 1: the packed kernel ran with the gap penalties patched in as
                          instruction immediates; 0: runtime operands */
    int32_t devices;   /* device entries that ran bands (band-cyclic multi-GPU Stage 1) */
    int32_t sp_slots;  /* special-row ring slots per unit (= the row count when all stayed resident) */
    int32_t tail_alpha, tail_warps, tail_grid; /* tail segment geometry (0: none; alpha < 0: packed) */
    int64_t tail_rows; /* rows of the tail segment */
} sw_stats;

/* Create a context on n_devices in {1, 2, 4, 8} CUDA devices.
 * device_ids[0] is the primary device: the reverse pass, Stage 2 and Stages
 * 3-5 run there.  With n_devices > 1, Stage 1 (sw_align_stage1*) runs as one
 * band pipeline across the devices (band-cyclic: device d takes bands d,
 * d + n, ...; each band's bottom row goes to the next device by peer stores
 * over NVLink), or as column stripes (sw_set_multi_gpu); the
 * library combines the per-device best cells under the total order of reading
 * S4 and hands the sink whole special rows.  Peer access is enabled between
 * every pair of distinct devices (SW_EINVAL if a pair has no P2P path).  An id
 * may repeat ("virtual peers" on one GPU, for testing): its entries share that
 * GPU's SMs.  Allocates the library's streams.  Returns SW_EINVAL / SW_ECUDA. */
int sw_init(const int *device_ids, int n_devices, sw_ctx **out);

/* Number of device entries of the context (sw_init's n_devices). */
int sw_device_count(const sw_ctx *ctx);

/* Multi-device Stage-1 partition (testing / tuning; default 1).  cyclic = 1:
 * band-cyclic rows (one pipeline of every device's CTAs); 0: the virtual
 * column stripes of one device (the entries beyond the first idle).
 * SW_EINVAL outside {0, 1}. */
int sw_set_multi_gpu(sw_ctx *ctx, int cyclic);

/* Total order of best cells (reading S4: higher score, then smaller i, then
 * smaller j; (0, 0, 0) when every score is 0) over `count` results, e.g. the
 * per-rank results of a multi-process stripe run.  SW_EINVAL on NULL. */
int sw_combine_best(const sw_result *results, int count, sw_result *out);

/* Stage 1 on host sequences.
 *   seqA : S0, m bytes of ACGTacgt (not NUL-terminated, borrowed for the call)
 *   seqB : S1, n bytes
 *   special_row_interval k >= 0: rows k, 2k, ... <= m go to `sink` (0 = none;
 *   any k >= 1 is correct, multiples of sw_row_granularity() are fastest).
 *   sink may be NULL when k == 0.
 *   out  : best score and end cell.
 * m or n == 0 returns {0,0,0} and no rows.  m, n < 2^31. */
int sw_align_stage1(sw_ctx *ctx, const char *seqA, int64_t m, const char *seqB, int64_t n,
                    int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
                    int64_t special_row_interval, sw_row_sink sink, void *user, sw_result *out);

/* Same as sw_align_stage1 but the sequences are DEVICE pointers (bytes of
 * ACGTacgt already resident in HBM on the context's device) and the work is
 * launched on `stream` (a cudaStream_t, or NULL for the library stream), so
 * the caller's CUDA events on that stream bracket the kernels.  Special-row
 * copies use the library's side stream.  Returns when the result is on the host. */
int sw_align_stage1_dev(sw_ctx *ctx, const char *dseqA, int64_t m, const char *dseqB, int64_t n,
                        int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
                        int64_t special_row_interval, sw_row_sink sink, void *user, void *stream,
                        sw_result *out);

/* Reverse pass (readings S9, S10): run the global
 * recurrence over S0[1..i_end]^R x S1[1..j_end]^R from H(0,0) = 0 and return
 * the first cell (i', j') (row-major, i', j' >= 1) whose H equals `goal`,
 * mapped to the forward start cell (i_end - i', j_end - j').  goal == 0
 * returns (0, i_end, j_end).  start_out = {goal, i_s, j_s}.
 * SW_ENOTFOUND when no cell equals goal. */
int sw_reverse_goal(sw_ctx *ctx, const char *seqA, int64_t i_end, const char *seqB, int64_t j_end,
                    int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
                    int32_t goal, sw_result *start_out);

/* sw_reverse_goal on DEVICE pointers (bytes of ACGTacgt resident in HBM),
 * kernels launched on `stream` (a cudaStream_t, or NULL for the library's). */
int sw_reverse_goal_dev(sw_ctx *ctx, const char *dseqA, int64_t i_end, const char *dseqB, int64_t j_end,
                        int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
                        int32_t goal, void *stream, sw_result *start_out);

/* Stage 2, partial traceback (readings S18-S22).
 * From the end point `end` (the Stage-1 result) back to the start point, find
 * where the optimal alignment crosses each special row by goal-based matching
 * of a reverse global fill against the special rows, which must still
 * be resident from the LAST sw_align_stage1 / sw_align_stage1_dev call on this
 * context with the same sequences, m, n, scoring and special_row_interval, run
 * on one GPU without virtual stripes (else SW_EINVAL; the sequences themselves
 * are the caller's responsibility).  special_row_interval 0 is allowed (one
 * partition: the start point only).
 * Output: the crosspoint list L_2 in ascending order, start point
 * first and `end` last, into out[0 .. cap) (caller-owned); *count = its
 * length.  cap < *count: the first cap entries are written and SW_ERANGE is
 * returned.  SW_ENOTFOUND when no junction exists (inputs inconsistent with
 * the rows).  The sequences are host pointers; the device variant below takes
 * HBM pointers and a stream. */
int sw_stage2(sw_ctx *ctx, const char *seqA, int64_t m, const char *seqB, int64_t n,
              int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
              int64_t special_row_interval, const sw_result *end,
              sw_crosspoint *out, int64_t cap, int64_t *count);

int sw_stage2_dev(sw_ctx *ctx, const char *dseqA, int64_t m, const char *dseqB, int64_t n,
                  int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
                  int64_t special_row_interval, const sw_result *end, void *stream,
                  sw_crosspoint *out, int64_t cap, int64_t *count);

/* One maximal gap run of the final alignment: (i, j) is the DP cell
 * the run leaves from (reading S24), len the number of gap columns.  GAP_1
 * holds gaps in S0 (horizontal: S1 characters against '-'), GAP_2 gaps in S1
 * (vertical). */
typedef struct {
    int64_t i;
    int64_t j;
    int64_t len;
} sw_gap;

/* The optimal local alignment: score, start cell (i0, j0) (the cell
 * before the first aligned pair, reading S8), end cell (i1, j1) (Stage 1's best
 * cell), the lengths of the GAP_1 / GAP_2 lists, and how the Myers-Miller stage
 * ran (partitions aligned in Stage 5, splitting levels). */
typedef struct {
    int32_t score;
    int64_t i0, j0, i1, j1;
    int64_t n_gap1, n_gap2;
    int64_t partitions, mm_levels;
    double ms_stage1, ms_stage2, ms_mm, ms_stage5;  /* host wall time per stage (Stages 3-4 = ms_mm) */
} sw_alignment;

/* Stages 1-5: the full optimal local alignment of S0 and S1.
 * Stage 1 with special rows every special_row_interval rows (0: none, one
 * Stage-2 partition), Stage 2 (crosspoints on the special rows, sw_stage2),
 * then Myers-Miller with balanced splitting on the GPU until every partition
 * has at most 65,536 cells, a full traceback of each, and the concatenation.
 * Sequences and scoring as sw_align_stage1; gap1[0 .. cap1) / gap2[0 .. cap2)
 * are caller-owned output arrays.  Returns SW_OK, or SW_ERANGE when a list did
 * not fit (out->n_gap1 / n_gap2 hold the lengths needed; the first cap
 * entries are written), or the errors of sw_align_stage1 / sw_stage2.
 * Alignments tie-break among optimal ones by the traceback preference
 * (diagonal, then vertical, then horizontal) inside each final partition. */
int sw_align(sw_ctx *ctx, const char *seqA, int64_t m, const char *seqB, int64_t n,
             int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
             int64_t special_row_interval, sw_alignment *out,
             sw_gap *gap1, int64_t cap1, sw_gap *gap2, int64_t cap2);

/* Rows per thread strip (alpha): special_row_interval multiples of this take
 * the fast special-row path. */
int64_t sw_row_granularity(const sw_ctx *ctx);

/* Rows per band (alpha x 32 x warps): the unit of the band pipeline and of the
 * multi-GPU border hand-off. */
int64_t sw_band_height(const sw_ctx *ctx);

/* Kernel selection (testing / tuning).  variant = -1: automatic choice per
 * call; 0..7: a fixed geometry (alpha, warps, tile width) of
 * the int32 kernel (DESIGN.md 4.1 lists them), or of the packed 16x2 kernel when packed = 1 and the call
 * qualifies (local mode, k % alpha == 0, small value window); 8..14: packed-only
 * geometries (alpha 32; 30 for 13; 34 x 8 warps for 14) that fall back to the default int32
 * geometry when the call does not qualify.  packed = 0 never uses the packed
 * kernel.  Results are identical for every choice.  SW_EINVAL outside -1..14. */
int sw_set_kernel(sw_ctx *ctx, int variant, int packed);

/* Immediate patching of the packed kernel (testing / tuning; default on).
 * on = 1: the packed kernel runs from a copy of its cubin whose gap-penalty
 * immediates are patched with the call's values, loaded once
 * per (gap_open, gap_ext) and context; on = 0: the kernel that reads them from
 * registers.  Results are identical; sw_stats.patched says which one ran.
 * Returns SW_EINVAL for a NULL ctx or on outside {0, 1}. */
int sw_set_patch(sw_ctx *ctx, int on);

/* Persistent-grid cap (testing / tuning; default 0).  ctas > 0: every fill
 * launch of the following calls runs at most `ctas` CTAs (at least one per
 * stripe) instead of the resident capacity, so bands outnumber CTAs and each
 * CTA takes several bands from the ticket (the band pipeline's multi-wave
 * path, P:134's grid of blocks over an arbitrary number of rows).  Results are
 * identical for every value.  SW_EINVAL for a NULL ctx or ctas < 0. */
int sw_set_grid(sw_ctx *ctx, int ctas);

/* Tail segment of a multi-wave Stage-1 fill (testing /
 * tuning).  mode -1 (default): automatic -- when the last wave of bands is
 * partial, the rows after the last full wave run as a second launch with a
 * shorter band height, if the band-pipeline model says it is faster; 0: never;
 * v + 1 (v a packed geometry of sw_set_kernel with a shorter band): always
 * that geometry when the fill has a partial last wave.  Results are identical.
 * SW_EINVAL outside -1 .. 15. */
int sw_set_tail(sw_ctx *ctx, int mode);

/* Device-memory budget of the special-row ring in bytes (testing / tuning;
 * 0 = default, 80 % of the free HBM).  Special rows that do not all fit stay
 * in a ring of as many slots as the budget holds (at least one band's rows);
 * a band waits for its slots until the host has copied the rows that used them
 * (back-pressure, P:178's bounded SRA), and the library keeps the rows in a
 * host store for Stage 2.  Any k >= 1 runs under any budget.
 * SW_EINVAL for bytes < 0. */
int sw_set_row_budget(sw_ctx *ctx, int64_t bytes);

/* ---- Column-stripe pipeline ----
 * The matrix is split into column stripes; stripe g sweeps every band of its
 * columns and hands the band's right-edge (t = H - G_first, E) column to stripe
 * g+1, per (band, warp), with a release flag carrying the call's epoch.
 *
 * Virtual stripes on one GPU (testing / small m): the next sw_align_stage1*
 * calls split [0, n) into `nstripes` (1..8) stripes run by one launch. */
int sw_set_virtual_stripes(sw_ctx *ctx, int nstripes);

/* One process per GPU.  Every rank except the first allocates its left-border
 * receive area for up to `max_rows` rows and exports it as a CUDA IPC handle
 * (64 bytes written to handle_out); the caller ships it to the left
 * neighbour (e.g. torch.distributed).  The left neighbour maps it with
 * sw_stripe_connect (NULL handle = last stripe).  Both must use the same band
 * height (same library build and variant). */
int sw_stripe_export(sw_ctx *ctx, int64_t max_rows, void *handle_out);
int sw_stripe_connect(sw_ctx *ctx, const void *right_handle, int64_t max_rows);

/* Highest epoch this context has run a stripe call with (0: none).  A group
 * of ranks agrees on the next epoch as 1 + the maximum over its ranks, so a
 * new group on a reused context never repeats an epoch its receive area has
 * seen. */
int32_t sw_stripe_epoch(const sw_ctx *ctx);

/* The kernel geometry the next rank call with these arguments would run
 * (alpha < 0: the packed kernel; warps per CTA): world = 0 for a column-stripe
 * rank (sw_align_stage1_stripe), else the band-cyclic group size
 * (sw_align_stage1_cyclic).  Ranks of one group must agree on it (band height
 * and border flags), which the caller checks before the call. */
int sw_plan(sw_ctx *ctx, int64_t m, int64_t n, int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
            int64_t special_row_interval, int32_t world, int32_t *alpha, int32_t *warps);

/* Stage 1 on this rank's stripe: global columns [c_lo, c_hi) of S1 (0-based),
 * all m rows.  dseqA / dseqB are the WHOLE sequences in this device's memory.
 * `epoch` must be the same on all ranks for one alignment and above
 * sw_stripe_epoch() of every rank (else SW_EINVAL).  `sink` receives this stripe's slice of each special row:
 * H, F = columns c_lo+1 .. c_hi, n = c_hi - c_lo.  `out` is this stripe's best
 * (score, i, j) in global coordinates; the global best is the maximum over
 * ranks under the same order (score, then smallest i, then smallest j). */
int sw_align_stage1_stripe(sw_ctx *ctx, const char *dseqA, int64_t m, const char *dseqB, int64_t n,
                           int64_t c_lo, int64_t c_hi, int32_t epoch,
                           int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
                           int64_t special_row_interval, sw_row_sink sink, void *user, void *stream,
                           sw_result *out);

/* ---- Band-cyclic ranks (one process per GPU) ----
 * Rank r of `world` runs bands r, r + world, ... of every row; band b reads its
 * top border (the row border and band b-1's progress) from this rank's
 * incoming area and stores its bottom row and progress into the next rank's
 * ((r + 1) mod world) area by peer stores over NVLink.  Each rank's sink gets
 * the WHOLE special rows of its own bands (ascending); `out` is the rank's
 * best (score, i, j) -- combine the ranks' with sw_combine_best.
 *
 * sw_cyclic_export allocates this rank's incoming area for up to max_rows x
 * max_cols and writes its 64-byte CUDA IPC handle; sw_cyclic_connect maps the
 * next rank's.  `epoch` must be the same on every rank of one call and above
 * sw_cyclic_epoch() of every rank (the areas' progress words are tagged with
 * it and never re-zeroed), else SW_EINVAL. */
int sw_cyclic_export(sw_ctx *ctx, int64_t max_rows, int64_t max_cols, void *handle_out);
int sw_cyclic_connect(sw_ctx *ctx, const void *next_handle, int64_t max_rows, int64_t max_cols);
int32_t sw_cyclic_epoch(const sw_ctx *ctx);
int sw_align_stage1_cyclic(sw_ctx *ctx, const char *dseqA, int64_t m, const char *dseqB, int64_t n,
                           int32_t rank, int32_t world, int32_t epoch,
                           int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
                           int64_t special_row_interval, sw_row_sink sink, void *user, void *stream,
                           sw_result *out);

/* Flush-interval rule of P:178 as a helper: the special-row spacing in rows,
 * R = bh * ceil(8 m n / (bh * sra_bytes)), for a byte budget sra_bytes. */
int64_t sw_special_row_interval_for_budget(int64_t m, int64_t n, int64_t bh, int64_t sra_bytes);

/* Stats of the last successful call on this context. */
int sw_get_stats(const sw_ctx *ctx, sw_stats *out);

/* Release everything.  NULL is a no-op. */
void sw_shutdown(sw_ctx *ctx);

/* Static description of an error code. */
const char *sw_strerror(int code);

/* Text of the last CUDA error seen on this context (empty if none). */
const char *sw_last_error(const sw_ctx *ctx);

#ifdef __cplusplus
}
#endif
#endif /* CUDALIGN_B200_H */
