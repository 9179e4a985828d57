// sw_api.cu -- C ABI (include/cudalign_b200.h) and host runtime of the
// B200-native Stage-1 engine: parameter validation, sequence encode/pack,
// persistent fill launch, special-row streaming to the host sink through
// pinned memory on a side stream, best-cell reduction, the
// reverse goal pass, and the column-stripe pipeline (one stripe
// per GPU over CUDA IPC / NVLink, or several virtual stripes on one GPU).
// No CPU fallback: every step runs in the kernels below or in sw_fill.cuh.
#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <unistd.h>
#include <vector>

#include "../../include/cudalign_b200.h"
#include "sw_fill.cuh"
#include "sw_fill16.cuh"

using namespace swb;

// ---------------------------------------------------------------- small device kernels

// a1: ASCII -> 2-bit codes (A=0, C=1, G=2, T=3, case-insensitive, reading S7),
// 16 codes per 32-bit word; optional reversal (reverse pass).  Any other byte
// sets *err.
__global__ void sw_encode_kernel(const unsigned char *sa, long long la, int reva, uint32_t *da, long long wa,
                                 const unsigned char *sb, long long lb, int revb, uint32_t *db, long long wb,
                                 int *err)
{
    long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const unsigned char *src;
    long long len;
    int rev;
    uint32_t *dst;
    if (w < wa) {
        src = sa; len = la; rev = reva; dst = da;
    } else {
        w -= wa;
        if (w >= wb) return;
        src = sb; len = lb; rev = revb; dst = db;
    }
    uint32_t word = 0;
    int bad = 0;
#pragma unroll
    for (int x = 0; x < 16; x++) {
        const long long i = w * 16 + x;
        if (i < len) {
            const unsigned char ch = src[rev ? len - 1 - i : i] | 0x20;
            uint32_t code = 0;
            if (ch == 'a') code = 0;
            else if (ch == 'c') code = 1;
            else if (ch == 'g') code = 2;
            else if (ch == 't') code = 3;
            else bad = 1;
            word |= code << (2 * x);
        }
    }
    dst[w] = word;
    if (bad) atomicOr(err, 1);
}

// a5: final (score, i, j) over the per-CTA slots (LOCAL), or decode the first
// hit (GLOBAL).  out = {score, i, j, status}.
__global__ void sw_reduce_kernel(const int4 *slots, int nslots, int local, const unsigned long long *hit_key,
                                 int goal, int4 *out)
{
    __shared__ int4 red[32];
    const int tid = threadIdx.x;
    if (!local) {
        if (tid == 0) {
            const unsigned long long k = *hit_key;
            if (k == ~0ull) *out = make_int4(goal, 0, 0, 0);
            else *out = make_int4(goal, (int)(k >> 32), (int)(k & 0xffffffffu), 1);
        }
        return;
    }
    int bs = 0, bi = 0, bj = 0;
    for (int x = tid; x < nslots; x += blockDim.x) {
        const int4 v = slots[x];
        if (v.x > 0 && better(v.x, v.y, v.z, bs, bi, bj)) { bs = v.x; bi = v.y; bj = v.z; }
    }
    for (int o = 16; o > 0; o >>= 1) {
        const int s2 = __shfl_down_sync(0xffffffffu, bs, o);
        const int i2 = __shfl_down_sync(0xffffffffu, bi, o);
        const int j2 = __shfl_down_sync(0xffffffffu, bj, o);
        if (s2 > 0 && better(s2, i2, j2, bs, bi, bj)) { bs = s2; bi = i2; bj = j2; }
    }
    if ((tid & 31) == 0) red[tid >> 5] = make_int4(bs, bi, bj, 0);
    __syncthreads();
    if (tid == 0) {
        int4 r = make_int4(0, 0, 0, 1);
        for (int w = 0; w < (int)(blockDim.x + 31) / 32; w++)
            if (red[w].x > 0 && better(red[w].x, red[w].y, red[w].z, r.x, r.y, r.z)) r = make_int4(red[w].x, red[w].y, red[w].z, 1);
        *out = r;
    }
}

// ---------------------------------------------------------------- kernel variants

struct Variant {
    int alpha, nw, w;
    const void *local_fn, *global_fn;
    size_t smem;
    const void *packed_fn;  // packed 16x2 Stage-1 kernel with the same band geometry (alpha 16 only)
    size_t smem16;
    int io_warps;           // 1, or 0 for the cooperative-I/O packed kernel (block = (nw + io) warps)
    int skew_tiles;         // int32 kernel: tiles past the last column lane 31 needs (ceil(62 / W))
    char packed_name[96];   // mangled name of the packed kernel in the patchable cubin ("" : none)
    const void *packed_global_fn;  // packed kernel in global (reverse-pass) mode, alpha 32 x 8 warps only
    char packed_global_name[96];
    const void *packed_gen_fn;  // packed kernel with the generic special-row tiles (GEN, sw_fill16.cuh)
    char packed_gen_name[96];
    const void *local_wide_fn, *global_wide_fn;  // int32 kernels for scorings outside the int8 profile (default geometry)
};

template <int NW, int W, bool COOP, int NS>
static void packed_name(Variant &v)
{
    snprintf(v.packed_name, sizeof(v.packed_name), "_ZN3swb16sw_fill16_kernelILi%dELi%dELb%dELi%dELb0ELb1ELb0EEEvNS_8FillArgsE",
             NW, W, COOP ? 1 : 0, NS);
}

// the GEN instantiation (generic special rows) of a packed geometry
template <int NW, int W, int NS>
static void packed_gen(Variant &v)
{
    v.packed_gen_fn = (const void *)&sw_fill16_kernel<NW, W, false, NS, false, true, true>;
    snprintf(v.packed_gen_name, sizeof(v.packed_gen_name),
             "_ZN3swb16sw_fill16_kernelILi%dELi%dELb0ELi%dELb0ELb1ELb1EEEvNS_8FillArgsE", NW, W, NS);
}

template <int ALPHA, int NW, int W, bool COOP = false, bool SPLIT = false>
static Variant make_variant()
{
    Variant v;
    v.alpha = ALPHA;
    v.nw = NW;
    v.w = W;
    v.local_fn = v.global_fn = nullptr;
    v.smem = 0;
    v.packed_fn = nullptr;
    v.smem16 = 0;
    v.io_warps = 1;
    v.skew_tiles = 1;
    v.packed_name[0] = 0;
    v.packed_global_fn = nullptr;
    v.packed_global_name[0] = 0;
    v.packed_gen_fn = nullptr;
    v.packed_gen_name[0] = 0;
    v.local_wide_fn = v.global_wide_fn = nullptr;
    if constexpr (ALPHA >= 30) {
        // packed kernel only (15 or 16 slots per lane); int32 work falls back to the default geometry
        constexpr int NS = ALPHA / 2;
        v.packed_fn = (const void *)&sw_fill16_kernel<NW, W, COOP, NS, SPLIT>;
        v.io_warps = COOP ? 0 : 1;
        v.smem16 = Fill16<NW, W, NS, SPLIT>::smem_bytes();
        if constexpr (!SPLIT) packed_name<NW, W, COOP, NS>(v);
        if constexpr (!SPLIT && !COOP) packed_gen<NW, W, NS>(v);  // variants 8, 10, 13, 14
        if constexpr (ALPHA == 32 && NW == 8 && !COOP && !SPLIT) {
            // the reverse pass (a8) on the packed kernel
            v.packed_global_fn = (const void *)&sw_fill16_kernel<NW, W, false, 16, false, false>;
            snprintf(v.packed_global_name, sizeof(v.packed_global_name),
                     "_ZN3swb16sw_fill16_kernelILi%dELi%dELb0ELi16ELb0ELb0ELb0EEEvNS_8FillArgsE", NW, W);
        }
        return v;
    } else {
        v.local_fn = (const void *)&sw_fill_kernel<ALPHA, NW, W, true>;
        v.global_fn = (const void *)&sw_fill_kernel<ALPHA, NW, W, false>;
        if constexpr (ALPHA == 16 && NW == 8 && W == 64) {
            v.local_wide_fn = (const void *)&sw_fill_kernel<ALPHA, NW, W, true, true>;
            v.global_wide_fn = (const void *)&sw_fill_kernel<ALPHA, NW, W, false, true>;
        }
        v.smem = Fill<ALPHA, NW, W, true>::smem_bytes();
        v.skew_tiles = (Fill<ALPHA, NW, W, true>::SKEW + W - 1) / W;
    }
    if constexpr (ALPHA == 16 && W % 64 == 0) {
        if constexpr (NW == 16) {
            v.packed_fn = (const void *)&sw_fill16_kernel<NW, W, true>;
            v.io_warps = 0;
            packed_name<NW, W, true, 8>(v);
        } else {
            v.packed_fn = (const void *)&sw_fill16_kernel<NW, W>;
            packed_name<NW, W, false, 8>(v);
            if constexpr (NW == 4 || NW == 8) packed_gen<NW, W, 8>(v);  // variants 0, 1
            if constexpr (NW == 8) {
                // Stage-2 partitions (global mode with matching) on the packed kernel
                v.packed_global_fn = (const void *)&sw_fill16_kernel<NW, W, false, 8, false, false>;
                snprintf(v.packed_global_name, sizeof(v.packed_global_name),
                         "_ZN3swb16sw_fill16_kernelILi%dELi%dELb0ELi8ELb0ELb0ELb0EEEvNS_8FillArgsE", NW, W);
            }
        }
        v.smem16 = Fill16<NW, W>::smem_bytes();
    }
    return v;
}

static constexpr int DEFAULT_VARIANT = 1;  // (alpha 16, 8 warps, W 64): fastest on C2/C3
static constexpr int NVARIANTS = 15;
static constexpr int NINT32_VARIANTS = 8;
// Dynamic shared memory the tail launch requests: more than
// half an SM's 228 KB, so its CTAs take one SM each as the main launch frees them.
static constexpr int TAIL_SMEM = 120 * 1024;  // variants 0..7 have int32 kernels; 8.. are packed-only (alpha 32)

static const Variant &variant_for(int idx)
{
    static const Variant vs[NVARIANTS] = {
        make_variant<16, 4, 64>(),
        make_variant<16, 8, 64>(),
        make_variant<8, 8, 64>(),
        make_variant<16, 12, 64>(),
        make_variant<16, 14, 64>(),
        make_variant<16, 15, 64>(),
        make_variant<16, 16, 64>(),
        make_variant<16, 8, 32>(),
        make_variant<32, 4, 64>(),
        make_variant<32, 4, 64, true>(),
        make_variant<32, 8, 64>(),
        make_variant<32, 16, 64, true>(),
        make_variant<32, 4, 64, false, true>(),  // split F chain (latency-bound one-wave fills)
        make_variant<30, 4, 64>(),  // 3840-row bands: one-wave matrices of up to 148 bands (C2: 142)
        make_variant<34, 8, 64>(),  // 8704-row bands: C4 as one wave of 8 x 148 CTAs (band-cyclic)
    };
    return vs[idx < 0 ? 0 : idx >= NVARIANTS ? NVARIANTS - 1 : idx];
}

// ---------------------------------------------------------------- context

struct DevBuf {
    void *p = nullptr;
    size_t cap = 0;
};

struct HostBuf {
    void *p = nullptr;
    size_t cap = 0;
    bool mapped = false;
};

// Border receive area of one stripe: (t, E) per DP row, then per (band, warp) epoch flags.
struct RecvArea {
    void *base = nullptr;  // device allocation (IPC-exportable)
    size_t rows = 0, flags = 0;
    int2 *lb() const { return (int2 *)base; }
    int *lready() const { return (int *)((char *)base + rows * sizeof(int2)); }
};

// Where the special rows of the last Stage-1 call live (for Stage 2): in the
// device ring (every row resident when the ring never wrapped), else in the
// library's host store (the paper's SRA).
struct S1Rows {
    bool valid = false;
    bool resident = false;       // row q at sp[0] + q * stride (H[0..n), F at + ld)
    bool stored = false;         // row q in host_rows[q] (H[0..n), F[n..2n))
    int64_t m = 0, n = 0, k = 0;
    int32_t ma = 0, mi = 0, go = 0, ge = 0;
    int64_t ld = 0, stride = 0;
};

constexpr int MAX_DEV = 8;

// Device entries 1.. of a multi-device context (entry 0 is the context's own
// fields).  Entries may repeat a physical device ("virtual peers", testing):
// their CTAs then share the GPU, and each launch is capped to its share.
struct Peer {
    int device = 0;
    cudaStream_t stream = nullptr, side = nullptr;
    cudaEvent_t ev[4] = {};
    std::vector<cudaEvent_t> ev_row;
    DevBuf a2, b2, misc, slots;
    int4 *res_h = nullptr;
};

// ---------------------------------------------------------------- patched packed kernels
//
// The packed cell update is bound by register reads: an add
// whose constant is an instruction immediate reads one register, with the
// constant in a register three.  The gap penalties are runtime values, so the
// packed kernels are also built into a separate cubin (sw_fill16_patch.cu)
// with magic immediates; per (G_ext, G_first) the library copies that image,
// overwrites the immediates (32-bit field at byte 4 of each 16-byte SASS
// instruction) and loads it with cudaLibraryLoadData.  The build checks that
// every occurrence of the magic words is such a field (build.py).

#if defined(SWB_PATCH_EXTERN) && !defined(__CUDA_ARCH__)
// the image is embedded by a separate object (build.py: an .incbin of the cubin,
// assembled and linked next to this one, so both compile in parallel)
extern "C" const unsigned char swb_patch_cubin_begin[];
extern "C" const unsigned char swb_patch_cubin_end[];
static const unsigned char *patch_image() { return swb_patch_cubin_begin; }
static size_t patch_image_size() { return (size_t)(swb_patch_cubin_end - swb_patch_cubin_begin); }
#elif defined(SWB_PATCH_CUBIN) && !defined(__CUDA_ARCH__)
asm(".section .rodata\n"
    ".balign 16\n"
    "swb_patch_cubin_begin:\n"
    ".incbin \"" SWB_PATCH_CUBIN "\"\n"
    "swb_patch_cubin_end:\n"
    ".previous\n");
extern "C" const unsigned char swb_patch_cubin_begin[] __asm__("swb_patch_cubin_begin");
extern "C" const unsigned char swb_patch_cubin_end[] __asm__("swb_patch_cubin_end");
static const unsigned char *patch_image() { return swb_patch_cubin_begin; }
static size_t patch_image_size() { return (size_t)(swb_patch_cubin_end - swb_patch_cubin_begin); }
#else
static const unsigned char *patch_image() { return nullptr; }
static size_t patch_image_size() { return 0; }
#endif

struct PatchedSet {
    int ge = -1, gf = -1;
    cudaLibrary_t lib = nullptr;
    const void *fn[5][NVARIANTS] = {};  // [packed, int32 local, int32 global, packed global, packed GEN][variant]
};

// Offsets of the magic immediates in the embedded image (computed once).
constexpr int NMAGIC = 6;
struct PatchSites {
    std::vector<size_t> off[NMAGIC];
    bool ok = false;
};
static const PatchSites &patch_sites()
{
    static PatchSites ps = [] {
        PatchSites p;
        const unsigned char *img = patch_image();
        const size_t n = patch_image_size();
        if (!img || n < 16) return p;
        const uint32_t magic[NMAGIC] = {SWB_K_NGE2, SWB_K_NGF2, SWB_K_NGE16, SWB_K_NGF16, SWB_K_NGE1, SWB_K_NGF1};
        for (size_t o = 0; o + 4 <= n; o++) {
            uint32_t w;
            memcpy(&w, img + o, 4);
            for (int k = 0; k < NMAGIC; k++)
                if (w == magic[k]) {
                    if (o % 16 != 4) return p;  // not an instruction immediate: refuse to patch
                    p.off[k].push_back(o);
                }
        }
        p.ok = !p.off[0].empty() && !p.off[2].empty() && !p.off[3].empty();
        return p;
    }();
    return ps;
}

struct sw_ctx {
    int device = 0;
    int num_sms = 0;
    int ndev = 1;               // device entries (sw_init's n_devices)
    int share[MAX_DEV] = {1};   // entries on the same physical GPU as entry d (grid share)
    Peer peer[MAX_DEV - 1];     // entries 1 .. ndev-1
    cudaStream_t stream = nullptr, side = nullptr;
    cudaStream_t aux = nullptr; // tail-segment launches (device 0)
    cudaEvent_t ev[6] = {};
    cudaEvent_t ev_aux[2] = {};
    std::vector<cudaEvent_t> ev_row;  // one per staging slot: the slot's final copy is done
    int nstage = 2;
    DevBuf seq, a2, b2, misc, slots, dbg;
    DevBuf mm_parts, mm_scratch, mm_res, mm_codes, mm_moves, mm_err, mm_cnt;  // Stages 3-5
    DevBuf capbuf;  // Stage 2: (t, E) of every DP row at the special row's column
    DevBuf rowb[MAX_STRIPES], progress[MAX_STRIPES], sp[MAX_STRIPES];
    HostBuf flags[MAX_STRIPES];  // mapped pinned row_done flags per stripe
    HostBuf colp[MAX_STRIPES];   // mapped pinned per-band final-column counts per stripe
    HostBuf stage;               // pinned staging for one special row (H then F)
    RecvArea vrecv[MAX_STRIPES]; // receive areas of virtual stripes 1..S-1
    // multi-GPU stripe (one per process): own receive area (exported), right neighbour's (imported)
    RecvArea recv;
    void *right_base = nullptr;
    size_t right_rows = 0;
    int epoch = 0;
    int dbg_n = 0;
    int4 *res_h = nullptr;  // pinned: result + err + replays
    sw_stats stats{};
    char errbuf[512] = {0};
    int variant_override = -1;
    int grid_cap = 0;           // sw_set_grid: CTAs per fill launch (0 = resident capacity; testing)
    int tail_mode = -1;         // sw_set_tail: -1 automatic, 0 off, v >= 0 + 1: force variant v-1 for the tail
    int cyclic = 1;             // multi-device Stage 1: 1 band-cyclic, 0 column stripes
    size_t sp_budget = 0;       // sw_set_row_budget: device bytes for the special-row ring (0: 0.8 x free)
    int pepoch = 0;             // tag of the last call's band-progress words
    HostBuf released;           // mapped, portable: special rows 0 .. value-1 have left the device ring
    std::vector<std::vector<int32_t>> host_rows;  // host store of special rows (ring mode)
    DevBuf s2row;               // Stage 2: one special row uploaded from the host store
    int unit_dev[MAX_STRIPES] = {-1, -1, -1, -1, -1, -1, -1, -1};  // physical device of unit u's rowb / progress / sp / vrecv (-1: none)
    int stripe_epoch = 0;       // highest epoch of a rank-mode stripe call (sw_stripe_epoch)
    // band-cyclic ranks (sw_cyclic_*): this rank's incoming row border + band
    // progress (exported over CUDA IPC), and the next rank's (imported)
    void *cin = nullptr;
    size_t cin_cols = 0, cin_bands = 0;
    void *cout = nullptr;
    size_t cout_cols = 0, cout_bands = 0;
    int vstripes = 1;           // virtual stripes for the single-process calls
    S1Rows s1;                  // special rows resident from the last Stage-1 call
    int packed = 1;             // use the packed 16x2 Stage-1 kernel when its preconditions hold
    int patch = 1;              // use the immediate-patched packed kernels (SWB_PATCH=0: runtime operands)
    bool patch_warned = false;
    std::vector<PatchedSet> patched;  // loaded patched images, most recent last
    long long timeout_ns = 120ll * 1000000000ll;
};

static int cuda_fail(sw_ctx *c, cudaError_t e, const char *what)
{
    if (c) snprintf(c->errbuf, sizeof(c->errbuf), "%s: %s", what, cudaGetErrorString(e));
    return SW_ECUDA;
}

#define CK(call)                                                          \
    do {                                                                  \
        cudaError_t e_ = (call);                                          \
        if (e_ != cudaSuccess) return cuda_fail(ctx, e_, #call);          \
    } while (0)

static int grow(sw_ctx *ctx, DevBuf &b, size_t bytes)
{
    if (b.cap >= bytes && b.p) return SW_OK;
    if (b.p) cudaFree(b.p);
    b.p = nullptr;
    b.cap = 0;
    size_t want = std::max<size_t>(bytes, 256);
    cudaError_t e = cudaMalloc(&b.p, want);
    if (e != cudaSuccess) {
        cudaGetLastError();
        snprintf(ctx->errbuf, sizeof(ctx->errbuf), "cudaMalloc(%zu): %s", want, cudaGetErrorString(e));
        return SW_ENOMEM;
    }
    b.cap = want;
    return SW_OK;
}

static int grow_host(sw_ctx *ctx, HostBuf &b, size_t bytes, bool mapped)
{
    if (b.cap >= bytes && b.p) return SW_OK;
    if (b.p) cudaFreeHost(b.p);
    b.p = nullptr;
    b.cap = 0;
    // portable: the mapped flags are read by every device of a multi-device context
    if (cudaHostAlloc(&b.p, std::max<size_t>(bytes, 64), cudaHostAllocPortable | (mapped ? cudaHostAllocMapped : 0)) != cudaSuccess) {
        cudaGetLastError();
        snprintf(ctx->errbuf, sizeof(ctx->errbuf), "cudaHostAlloc(%zu) failed", bytes);
        return SW_ENOMEM;
    }
    b.cap = std::max<size_t>(bytes, 64);
    b.mapped = mapped;
    return SW_OK;
}

static int grow_recv(sw_ctx *ctx, RecvArea &r, size_t rows, size_t flags)
{
    if (r.base && r.rows >= rows && r.flags >= flags) return SW_OK;
    if (r.base) cudaFree(r.base);
    r.base = nullptr;
    const size_t bytes = rows * sizeof(int2) + flags * sizeof(int);
    if (cudaMalloc(&r.base, bytes) != cudaSuccess) {
        cudaGetLastError();
        snprintf(ctx->errbuf, sizeof(ctx->errbuf), "cudaMalloc(%zu) for a border area failed", bytes);
        return SW_ENOMEM;
    }
    cudaMemset(r.base, 0, bytes);  // flags start at epoch 0; calls use epochs >= 1
    r.rows = rows;
    r.flags = flags;
    return SW_OK;
}

extern "C" const char *sw_strerror(int code)
{
    switch (code) {
    case SW_OK: return "ok";
    case SW_EINVAL: return "invalid argument";
    case SW_EALPHABET: return "sequence byte outside ACGTacgt";
    case SW_ERANGE: return "scores could exceed the int32-safe range";
    case SW_ENOMEM: return "out of memory";
    case SW_ECUDA: return "CUDA error";
    case SW_EABORTED: return "aborted by the special-row sink";
    case SW_ENOTFOUND: return "no cell equals the goal score";
    default: return "unknown error";
    }
}

extern "C" const char *sw_last_error(const sw_ctx *ctx) { return ctx ? ctx->errbuf : ""; }

// Per-device view of a context entry (entry 0: the context's own fields).
struct DevView {
    int device;
    cudaStream_t stream, side;
    cudaEvent_t *ev;
    std::vector<cudaEvent_t> *ev_row;
    DevBuf *a2, *b2, *misc, *slots;
    int4 *res_h;
};
static DevView dview(sw_ctx *ctx, int d)
{
    if (d == 0)
        return DevView{ctx->device, ctx->stream, ctx->side, ctx->ev, &ctx->ev_row, &ctx->a2, &ctx->b2, &ctx->misc,
                       &ctx->slots, ctx->res_h};
    Peer &P = ctx->peer[d - 1];
    return DevView{P.device, P.stream, P.side, P.ev, &P.ev_row, &P.a2, &P.b2, &P.misc, &P.slots, P.res_h};
}

static void set_kernel_attrs()
{
    for (int i = 0; i < NVARIANTS; i++) {
        const Variant &v = variant_for(i);
        if (v.local_fn) cudaFuncSetAttribute(v.local_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem);
        if (v.local_wide_fn) cudaFuncSetAttribute(v.local_wide_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem);
        if (v.global_wide_fn) cudaFuncSetAttribute(v.global_wide_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem);
        if (v.global_fn) cudaFuncSetAttribute(v.global_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem);
        if (v.packed_fn) cudaFuncSetAttribute(v.packed_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, TAIL_SMEM);
        if (v.packed_global_fn)
            cudaFuncSetAttribute(v.packed_global_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem16);
        if (v.packed_gen_fn) cudaFuncSetAttribute(v.packed_gen_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, TAIL_SMEM);
    }
}

extern "C" int sw_init(const int *device_ids, int n_devices, sw_ctx **out)
{
    if (!out || !device_ids || !(n_devices == 1 || n_devices == 2 || n_devices == 4 || n_devices == 8)) return SW_EINVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev <= 0) { cudaGetLastError(); return SW_ECUDA; }
    for (int d = 0; d < n_devices; d++)
        if (device_ids[d] < 0 || device_ids[d] >= ndev) return SW_EINVAL;
    sw_ctx *ctx = new sw_ctx();
    ctx->device = device_ids[0];
    ctx->ndev = n_devices;
    for (int d = 1; d < n_devices; d++) ctx->peer[d - 1].device = device_ids[d];
    for (int d = 0; d < n_devices; d++) {
        ctx->share[d] = 0;
        for (int e = 0; e < n_devices; e++) ctx->share[d] += device_ids[e] == device_ids[d];
    }
    int rc = SW_OK;
    do {
        cudaError_t e;
        if ((e = cudaSetDevice(ctx->device)) != cudaSuccess) { rc = cuda_fail(ctx, e, "cudaSetDevice"); break; }
        cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, ctx->device);
        if ((e = cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking)) != cudaSuccess) { rc = cuda_fail(ctx, e, "stream"); break; }
        if ((e = cudaStreamCreateWithFlags(&ctx->side, cudaStreamNonBlocking)) != cudaSuccess) { rc = cuda_fail(ctx, e, "stream"); break; }
        if ((e = cudaStreamCreateWithFlags(&ctx->aux, cudaStreamNonBlocking)) != cudaSuccess) { rc = cuda_fail(ctx, e, "stream"); break; }
        for (auto &ev : ctx->ev)
            if ((e = cudaEventCreate(&ev)) != cudaSuccess) { rc = cuda_fail(ctx, e, "event"); break; }
        for (auto &ev : ctx->ev_aux)
            if ((e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)) != cudaSuccess) { rc = cuda_fail(ctx, e, "event"); break; }
        if (rc) break;
        if ((e = cudaHostAlloc(&ctx->res_h, 4 * sizeof(int4), cudaHostAllocDefault)) != cudaSuccess) { rc = SW_ENOMEM; break; }
        if (cudaHostAlloc(&ctx->released.p, 64, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) { rc = SW_ENOMEM; break; }
        ctx->released.cap = 64;
        ctx->released.mapped = true;
        set_kernel_attrs();
        if ((e = cudaGetLastError()) != cudaSuccess) { rc = cuda_fail(ctx, e, "cudaFuncSetAttribute"); break; }
        // entries 1..: streams, events and peer access in both directions with
        // every other physical device of the context (the band-cyclic pipeline
        // stores each band's bottom row into the next entry's memory)
        for (int d = 1; d < n_devices && !rc; d++) {
            Peer &P = ctx->peer[d - 1];
            if ((e = cudaSetDevice(P.device)) != cudaSuccess) { rc = cuda_fail(ctx, e, "cudaSetDevice(peer)"); break; }
            if ((e = cudaStreamCreateWithFlags(&P.stream, cudaStreamNonBlocking)) != cudaSuccess) { rc = cuda_fail(ctx, e, "stream"); break; }
            if ((e = cudaStreamCreateWithFlags(&P.side, cudaStreamNonBlocking)) != cudaSuccess) { rc = cuda_fail(ctx, e, "stream"); break; }
            for (auto &ev : P.ev)
                if ((e = cudaEventCreate(&ev)) != cudaSuccess) { rc = cuda_fail(ctx, e, "event"); break; }
            if (rc) break;
            if ((e = cudaHostAlloc(&P.res_h, 4 * sizeof(int4), cudaHostAllocDefault)) != cudaSuccess) { rc = SW_ENOMEM; break; }
            set_kernel_attrs();
        }
        for (int d = 0; d < n_devices && !rc; d++)
            for (int f = 0; f < n_devices && !rc; f++) {
                if (device_ids[d] == device_ids[f]) continue;
                int can = 0;
                cudaDeviceCanAccessPeer(&can, device_ids[d], device_ids[f]);
                if (!can) {
                    snprintf(ctx->errbuf, sizeof(ctx->errbuf), "device %d cannot access device %d (no P2P)", device_ids[d], device_ids[f]);
                    rc = SW_EINVAL;
                    break;
                }
                cudaSetDevice(device_ids[d]);
                e = cudaDeviceEnablePeerAccess(device_ids[f], 0);
                if (e == cudaErrorPeerAccessAlreadyEnabled) { cudaGetLastError(); e = cudaSuccess; }
                if (e != cudaSuccess) rc = cuda_fail(ctx, e, "cudaDeviceEnablePeerAccess");
            }
        cudaSetDevice(ctx->device);
        if (rc) break;
        if (const char *ov = getenv("SWB_VARIANT")) ctx->variant_override = atoi(ov);
        if (const char *vs = getenv("SWB_VSTRIPES")) ctx->vstripes = std::max(1, std::min(MAX_STRIPES, atoi(vs)));
        if (const char *to = getenv("SWB_TIMEOUT_S")) ctx->timeout_ns = (long long)(atof(to) * 1e9);
        if (const char *pk = getenv("SWB_PACKED")) ctx->packed = atoi(pk);
        if (const char *pt = getenv("SWB_PATCH")) ctx->patch = atoi(pt);
        if (const char *tl = getenv("SWB_TAIL")) ctx->tail_mode = atoi(tl);
    } while (0);
    if (rc) { sw_shutdown(ctx); return rc; }
    *out = ctx;
    return SW_OK;
}

extern "C" void sw_shutdown(sw_ctx *ctx)
{
    if (!ctx) return;
    for (int d = 1; d < ctx->ndev; d++) {
        Peer &P = ctx->peer[d - 1];
        if (cudaSetDevice(P.device) != cudaSuccess) continue;
        if (P.stream) cudaStreamSynchronize(P.stream);
        if (P.side) cudaStreamSynchronize(P.side);
        for (DevBuf *b : {&P.a2, &P.b2, &P.misc, &P.slots})
            if (b->p) cudaFree(b->p);
        if (P.res_h) cudaFreeHost(P.res_h);
        for (auto &ev : P.ev)
            if (ev) cudaEventDestroy(ev);
        for (auto &ev : P.ev_row)
            if (ev) cudaEventDestroy(ev);
        if (P.stream) cudaStreamDestroy(P.stream);
        if (P.side) cudaStreamDestroy(P.side);
    }
    cudaSetDevice(ctx->device);
    if (ctx->stream) cudaStreamSynchronize(ctx->stream);
    if (ctx->side) cudaStreamSynchronize(ctx->side);
    if (ctx->aux) cudaStreamSynchronize(ctx->aux);
    for (DevBuf *b : {&ctx->seq, &ctx->a2, &ctx->b2, &ctx->misc, &ctx->slots, &ctx->dbg, &ctx->capbuf, &ctx->mm_parts,
                      &ctx->mm_scratch, &ctx->mm_res, &ctx->mm_codes, &ctx->mm_moves, &ctx->mm_err, &ctx->mm_cnt, &ctx->s2row})
        if (b->p) cudaFree(b->p);
    for (int s = 0; s < MAX_STRIPES; s++) {
        cudaSetDevice(ctx->unit_dev[s] >= 0 ? ctx->unit_dev[s] : ctx->device);  // a unit's buffers live on its entry's device
        for (DevBuf *b : {&ctx->rowb[s], &ctx->progress[s], &ctx->sp[s]})
            if (b->p) cudaFree(b->p);
        if (ctx->flags[s].p) cudaFreeHost(ctx->flags[s].p);
        if (ctx->colp[s].p) cudaFreeHost(ctx->colp[s].p);
        if (ctx->vrecv[s].base) cudaFree(ctx->vrecv[s].base);
    }
    cudaSetDevice(ctx->device);
    for (auto &P : ctx->patched)
        if (P.lib) cudaLibraryUnload(P.lib);
    if (ctx->right_base) cudaIpcCloseMemHandle(ctx->right_base);
    if (ctx->cout) cudaIpcCloseMemHandle(ctx->cout);
    if (ctx->cin) cudaFree(ctx->cin);
    if (ctx->recv.base) cudaFree(ctx->recv.base);
    if (ctx->stage.p) cudaFreeHost(ctx->stage.p);
    if (ctx->released.p) cudaFreeHost(ctx->released.p);
    if (ctx->res_h) cudaFreeHost(ctx->res_h);
    for (auto &ev : ctx->ev)
        if (ev) cudaEventDestroy(ev);
    for (auto &ev : ctx->ev_aux)
        if (ev) cudaEventDestroy(ev);
    for (auto &ev : ctx->ev_row)
        if (ev) cudaEventDestroy(ev);
    if (ctx->stream) cudaStreamDestroy(ctx->stream);
    if (ctx->side) cudaStreamDestroy(ctx->side);
    if (ctx->aux) cudaStreamDestroy(ctx->aux);
    delete ctx;
}

// The geometry int32 work (reverse pass, Stage 2) runs with: the override when
// it has an int32 kernel, else the default.
static const Variant &ctx_variant(const sw_ctx *ctx)
{
    const int v = ctx->variant_override;
    return variant_for(v >= 0 && v < NINT32_VARIANTS ? v : DEFAULT_VARIANT);
}

extern "C" int64_t sw_row_granularity(const sw_ctx *ctx)
{
    if (!ctx) return 0;
    return variant_for(ctx->variant_override >= 0 ? ctx->variant_override : DEFAULT_VARIANT).alpha;
}

extern "C" int64_t sw_band_height(const sw_ctx *ctx)
{
    if (!ctx) return 0;
    const Variant &v = ctx_variant(ctx);
    return (int64_t)v.alpha * 32 * v.nw;
}

extern "C" int64_t sw_special_row_interval_for_budget(int64_t m, int64_t n, int64_t bh, int64_t sra_bytes)
{
    // Flush interval (blocks of bh rows) >= ceil(8 m n / (bh |SRA|)).
    if (m <= 0 || n <= 0 || bh <= 0 || sra_bytes <= 0) return 0;
    const unsigned __int128 num = (unsigned __int128)8 * (unsigned __int128)m * (unsigned __int128)n;
    const unsigned __int128 den = (unsigned __int128)bh * (unsigned __int128)sra_bytes;
    unsigned __int128 q = (num + den - 1) / den;
    if (q < 1) q = 1;
    return (int64_t)(bh * (int64_t)q);
}

extern "C" int sw_set_kernel(sw_ctx *ctx, int variant, int packed)
{
    if (!ctx || variant < -1 || variant >= NVARIANTS || packed < 0 || packed > 1) return SW_EINVAL;
    ctx->variant_override = variant;
    ctx->packed = packed;
    return SW_OK;
}

extern "C" int sw_set_patch(sw_ctx *ctx, int on)
{
    if (!ctx || on < 0 || on > 1) return SW_EINVAL;
    ctx->patch = on;
    return SW_OK;
}

extern "C" int sw_set_tail(sw_ctx *ctx, int mode)
{
    if (!ctx || mode < -1 || mode > NVARIANTS) return SW_EINVAL;
    ctx->tail_mode = mode;
    return SW_OK;
}

extern "C" int sw_set_row_budget(sw_ctx *ctx, int64_t bytes)
{
    if (!ctx || bytes < 0) return SW_EINVAL;
    ctx->sp_budget = (size_t)bytes;
    return SW_OK;
}

extern "C" int sw_set_multi_gpu(sw_ctx *ctx, int cyclic)
{
    if (!ctx || cyclic < 0 || cyclic > 1) return SW_EINVAL;
    ctx->cyclic = cyclic;
    return SW_OK;
}

extern "C" int sw_device_count(const sw_ctx *ctx) { return ctx ? ctx->ndev : 0; }

extern "C" int32_t sw_stripe_epoch(const sw_ctx *ctx) { return ctx ? ctx->stripe_epoch : 0; }

extern "C" int sw_combine_best(const sw_result *results, int count, sw_result *out)
{
    if (!out || count < 0 || (count > 0 && !results)) return SW_EINVAL;
    sw_result b{0, 0, 0};
    for (int x = 0; x < count; x++) {
        const sw_result &r = results[x];
        if (r.score <= 0) continue;
        if (r.score > b.score || (r.score == b.score && (r.i < b.i || (r.i == b.i && r.j < b.j)))) b = r;
    }
    *out = b;
    return SW_OK;
}

extern "C" int sw_set_grid(sw_ctx *ctx, int ctas)
{
    if (!ctx || ctas < 0) return SW_EINVAL;
    ctx->grid_cap = ctas;
    return SW_OK;
}

extern "C" int sw_set_virtual_stripes(sw_ctx *ctx, int nstripes)
{
    if (!ctx || nstripes < 1 || nstripes > MAX_STRIPES) return SW_EINVAL;
    ctx->vstripes = nstripes;
    return SW_OK;
}

// Debug: copy the per-band timestamps of the last fill (SWB_DEBUG_TIMES set).
extern "C" int64_t swb_debug_times(sw_ctx *ctx, unsigned long long *out, int64_t cap)
{
    if (!ctx || !ctx->dbg.p || !out) return 0;
    const int64_t n = std::min<int64_t>(cap, (int64_t)ctx->dbg_n * 80);
    cudaMemcpy(out, ctx->dbg.p, n * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
    return n;
}

extern "C" int sw_get_stats(const sw_ctx *ctx, sw_stats *out)
{
    if (!ctx || !out) return SW_EINVAL;
    *out = ctx->stats;
    return SW_OK;
}

// ---------------------------------------------------------------- validation

static int check_scoring(int32_t ma, int32_t mi, int32_t go, int32_t ge, int64_t m, int64_t n)
{
    if (go < 0 || ge < 0) return SW_EINVAL;
    const long long gf = (long long)go + ge;
    const long long lim = 1ll << 30;
    const long long mn = std::min(m, n);
    if (mn * (long long)std::max(std::abs(ma), std::abs(mi)) >= lim) return SW_ERANGE;
    if ((m + n + 2) * (gf + 1) + mn * (long long)std::abs(mi) >= lim) return SW_ERANGE;
    return SW_OK;
}

// ---------------------------------------------------------------- the core call

namespace {
struct Job {
    const unsigned char *dA;
    int64_t m;
    const unsigned char *dB;
    int64_t n;
    bool revA, revB;
    int32_t ma, mi, go, ge;
    int64_t k;
    sw_row_sink sink;
    void *user;
    bool local;
    int32_t goal;
    // Stage-2 partition: start-check width, anchor type, matching
    int hit_w = 0x7fffffff;
    bool anchor_gap = false;
    bool match = false;
    int64_t mjc = 0;
    const int *mH = nullptr, *mF = nullptr;
    // stripes: either `nv` virtual stripes of [0, n) on this GPU, or (rank mode)
    // one stripe [c_lo, c_hi) whose borders come from / go to other GPUs.
    int nv = 1;
    bool rank_mode = false;
    int64_t c_lo = 0, c_hi = 0;
    int epoch = 0;
    // scoring outside the int8 profile window (|p + G_first| > 127): the WIDE int32 kernels
    bool wide = false;
    // band-cyclic rank (one process per GPU): this rank runs bands rank, rank + world, ...
    bool rank_cyc = false;
    int cyc_world = 1, cyc_rank = 0;
};
}  // namespace

// Kernel choice per call: a small cost model over candidate
// (kernel, geometry) pairs -- the band pipeline recurrence below with each
// candidate's measured column speed per CTA (one B200,
// profiles/r01_variants.txt).  Deterministic in (m, n, k, scoring), so all
// ranks of a stripe group agree.
struct Candidate {
    int variant;
    bool packed;
    double cps_full;  // columns/s one CTA sweeps with every resident CTA busy (R10M x 1M, one B200)
    double cps_solo;  // columns/s of a CTA alone on its SM (C2: 133 bands on 148 SMs)
};

// profiles/r01_variants.txt; earlier entries win near-ties (3 %)
static const Candidate kCands[] = {
    {DEFAULT_VARIANT, false, 4.24e6, 4.24e6},  // int32, 8 warps + I/O warp
    {1, true, 8.08e6, 7.74e6},                 // packed alpha 16, 8 warps + I/O warp
    {8, true, 4.25e6, 7.86e6},                 // packed alpha 32, 4 warps + I/O warp (2 CTAs/SM)
    {13, true, 4.45e6, 8.17e6},                // packed alpha 30, 4 warps + I/O warp (2 CTAs/SM)
    {10, true, 4.49e6, 4.49e6},                // packed alpha 32, 8 warps + I/O warp
    {5, true, 4.03e6, 4.03e6},                 // packed alpha 16, 15 warps + I/O warp
    {6, true, 3.87e6, 3.87e6},                 // packed alpha 16, 16 warps, cooperative I/O
    {14, true, 4.49e6 * 32 / 34, 4.49e6 * 32 / 34},  // packed alpha 34, 8 warps + I/O warp
};
static constexpr int NCANDS = (int)(sizeof(kCands) / sizeof(kCands[0]));
// Tail-segment candidates: column speed of one CTA alone on
// its SM (the tail launch holds one CTA per SM).
static const Candidate kTailCands[] = {
    {0, true, 12.0e6, 12.0e6},   // packed alpha 16, 4 warps + I/O warp: 2048-row bands
    {13, true, 8.17e6, 8.17e6},  // packed alpha 30, 4 warps: 3840-row bands
    {8, true, 7.86e6, 7.86e6},   // packed alpha 32, 4 warps: 4096-row bands
    {1, true, 7.74e6, 7.74e6},   // packed alpha 16, 8 warps: 4096-row bands
};

// Modelled fill time of a candidate: band b starts when its CTA is free and
// band b-1 is `lag` columns ahead,
//   start(b) = max(start(b - P) + n / cps, start(b - 1) + lag / cps),
//   T = start(nb - 1) + n / cps,
// with P resident CTAs and lag = (2 NW + 2) W columns (NW warps skewed by two
// tiles, plus the border load one tile ahead and drain one tile behind).
static double model_fill_time(long long nb, long long P, long long n, long long lag, double cps)
{
    // closed form of the recurrence: the max is at the last full CTA sweep when n >= P lag
    const long long b = nb - 1;
    const double chain = (double)b * (double)lag;
    const double waves = (double)(b / P) * (double)n + (double)(b % P) * (double)lag;
    return (std::max(chain, waves) + (double)n) / cps;
}

// The patched packed kernel of variant V for (G_ext, G_first), loading the
// image on first use (at most 4 images per context, oldest unloaded first).
// nullptr: not available (no embedded image, SWB_PATCH=0, or a load error),
// and the caller runs the runtime-operand kernel (same results).
static const void *patched_kernel(sw_ctx *ctx, const Variant &V, int ge, int gf, int kind = 0)
{
    // kind 0: packed local, 3: packed global, 4: packed local GEN (the kernels in
    // the patched image); 1, 2: int32 local/global (not patched)
    if ((kind != 0 && kind != 3 && kind != 4) || !ctx->patch) return nullptr;
    const char *name = kind == 0 ? V.packed_name : kind == 3 ? V.packed_global_name : V.packed_gen_name;
    if (!name[0]) return nullptr;
    const PatchSites &ps = patch_sites();
    if (!ps.ok) return nullptr;
    const int vidx = (int)(&V - &variant_for(0));
    if (vidx < 0 || vidx >= NVARIANTS) return nullptr;
    PatchedSet *P = nullptr;
    for (auto &q : ctx->patched)
        if (q.ge == ge && q.gf == gf) P = &q;
    if (!P) {
        std::vector<unsigned char> img(patch_image(), patch_image() + patch_image_size());
        const uint32_t val[NMAGIC] = {(uint32_t)(-(ge * 0x10001)), (uint32_t)(-(gf * 0x10001)),
                                      ((0x10000u - (uint32_t)ge) & 0xffffu) * 0x10001u,
                                      ((0x10000u - (uint32_t)gf) & 0xffffu) * 0x10001u, (uint32_t)(-ge),
                                      (uint32_t)(-gf)};
        for (int k = 0; k < NMAGIC; k++)
            for (size_t o : ps.off[k]) memcpy(img.data() + o, &val[k], 4);
        PatchedSet q;
        q.ge = ge;
        q.gf = gf;
        if (cudaLibraryLoadData(&q.lib, img.data(), nullptr, nullptr, 0, nullptr, nullptr, 0) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        if (ctx->patched.size() >= 4) {
            cudaDeviceSynchronize();  // an older image may still run on a caller's stream
            cudaLibraryUnload(ctx->patched.front().lib);
            ctx->patched.erase(ctx->patched.begin());
        }
        ctx->patched.push_back(q);
        P = &ctx->patched.back();
    }
    if (!P->fn[kind][vidx]) {
        cudaKernel_t k = nullptr;
        if (cudaLibraryGetKernel(&k, P->lib, name) != cudaSuccess || !k) {
            cudaGetLastError();
            if (!ctx->patch_warned) {  // a name/instantiation mismatch: say so once, run unpatched
                fprintf(stderr, "[cudalign_b200] patched kernel %s not in the embedded image; using register operands\n", name);
                ctx->patch_warned = true;
            }
            return nullptr;
        }
        if (cudaFuncSetAttribute((const void *)k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)(kind == 0 || kind == 4 ? std::max<size_t>(V.smem16, TAIL_SMEM) : kind == 3 ? V.smem16 : V.smem)) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        P->fn[kind][vidx] = (const void *)k;
    }
    return P->fn[kind][vidx];
}

// The packed kernel's preconditions for a local-mode fill.
static bool packed_qualifies(const sw_ctx *ctx, const Job &J, const Variant &V)
{
    const long long pmax_abs = std::max(std::abs(J.ma), std::abs(J.mi));
    const long long span = 32ll * V.alpha + 140;
    // k >= alpha: at most one special row per lane; rows that are not strip
    // bottoms take the generic special-row tiles of the GEN instantiation (SPM 2,
    // sw_fill16.cuh; variants 0, 1, 8, 10, 13)
    const bool rows_ok = J.k == 0 || J.k % V.alpha == 0 || (J.k >= V.alpha && V.packed_gen_fn);
    return ctx->packed && J.local && V.packed_fn && rows_ok && span * (pmax_abs + J.go + J.ge) + 1024 < 30000;
}

static const Variant &choose_variant(sw_ctx *ctx, const Job &J, bool *use16, int gpus = 1)
{
    if (J.wide) {  // only the default int32 geometry has the WIDE instantiation
        *use16 = false;
        return variant_for(DEFAULT_VARIANT);
    }
    const long long pmax_abs = std::max(std::abs(J.ma), std::abs(J.mi));
    // packed preconditions: local mode, special rows at strip
    // bottoms, and a warp's live values (32 alpha rows x ~130 columns of
    // Manhattan distance, each step <= p_max + G_first apart) inside the 16-bit frame
    auto packed_ok = [&](const Variant &V) { return packed_qualifies(ctx, J, V); };
    if (!J.local && J.match && !J.anchor_gap && ctx->variant_override < 0) {
        // Stage-2 partitions: the packed kernel in global mode with the band-end
        // matching, alpha 16 x 8 warps (4096-row bands, the int32 default's
        // geometry: these one-wave fills stop after the band with the first event).
        // Gap anchors (S20) put -inf in column 0, outside the 16-bit frame: int32.
        const Variant &V = variant_for(1);
        const long long span = 32ll * V.alpha + 140;
        *use16 = ctx->packed && V.packed_global_fn && J.k == 0 && !J.rank_mode && J.nv == 1 &&
                 span * (pmax_abs + J.go + J.ge) + 1024 < 30000 && !(getenv("SWB_S2PACKED") && atoi(getenv("SWB_S2PACKED")) == 0);
        if (*use16) return V;
    }
    if (!J.local) {
        // reverse pass (a8): the packed kernel in global mode when it qualifies
        // (alpha 32 x 8 warps geometry; one stripe, no Stage-2 matching or gap anchor)
        const Variant &V = variant_for(10);
        const long long span = 32ll * V.alpha + 140;
        *use16 = ctx->packed && V.packed_global_fn && !J.match && !J.anchor_gap && J.k == 0 && !J.rank_mode &&
                 J.nv == 1 && (ctx->variant_override < 0 || ctx->variant_override == 10) &&
                 span * (pmax_abs + J.go + J.ge) + 1024 < 30000;
        if (*use16) return V;
    }
    if (ctx->variant_override >= 0) {
        const Variant &V = variant_for(ctx->variant_override);
        *use16 = packed_ok(V);
        if (!*use16 && !V.local_fn) return variant_for(DEFAULT_VARIANT);  // packed-only geometry
        return V;
    }
    const Candidate *cands = kCands;
    double best_t = 1e300;
    int best = 0;
    for (int c = 0; c < NCANDS; c++) {
        const Candidate &C = cands[c];
        const Variant &V = variant_for(C.variant);
        if (C.packed && !packed_ok(V)) continue;
        // alpha 34 (variant 14) is for band-cyclic fills on several GPUs (one wave
        // of 8 x 148 CTAs on C4); on one GPU alpha 32 + the tail launch is faster
        if (C.variant == 14 && gpus == 1) continue;
        if (!C.packed && !J.local) { best = c; break; }  // reverse pass: int32 only
        const void *fn = C.packed ? V.packed_fn : V.local_fn;
        if (!fn) continue;
        int per_sm = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, V.nw * 32 + (C.packed ? V.io_warps : 1) * 32,
                                                      C.packed ? V.smem16 : V.smem);
        // band-cyclic multi-GPU: one pipeline of `gpus` x the resident CTAs
        const long long P = (long long)std::max(1, per_sm) * ctx->num_sms * gpus;
        const long long bh = (long long)V.alpha * 32 * V.nw;
        const long long nb = std::max<long long>(1, (J.m + bh - 1) / bh);
        const double cps = nb <= (long long)ctx->num_sms * gpus ? C.cps_solo : C.cps_full;
        double t = model_fill_time(nb, P, std::max<long long>(J.n, 1), (2ll * V.nw + 2) * V.w, cps);
        // special rows that are not band bottoms are written by the compute
        // warps (SP1 tiles) instead of the I/O warp: measured +7.7 % on C2
        // (variant 8 at k = 3840 vs 4096, profiles/r01_fill_a30.txt)
        // (profiles/r02_spm3.txt: 1.099 at strip bottoms, 1.049 for one staged
        // row per band, k >= bh; several generic rows per band run the
        // per-slot select path: C3 at k = 4096 on alpha 34 was 5x slower)
        if (J.k > 0 && J.k < J.m && J.k % bh != 0) t *= J.k % V.alpha == 0 ? 1.099 : J.k >= bh ? 1.049 : 4.0;
        if (t < best_t * 0.97) {
            best_t = t;
            best = c;
        }
    }
    *use16 = cands[best].packed;
    return variant_for(cands[best].variant);
}

// One fill SEGMENT: a launch (per device entry) of one kernel geometry over
// rows [row_base, row_base + nb BH).
struct Seg {
    const Variant *V = nullptr;
    bool use16 = false;
    int row_base = 0, band_base = 0, nb = 0, BH = 0;
    const void *fn = nullptr;
    size_t smem = 0;
    int block = 0;
    bool patched = false;
    int grid[MAX_DEV] = {};
};

static bool distinct_devices(const sw_ctx *ctx)
{
    for (int d = 1; d < ctx->ndev; d++)
        if (ctx->peer[d - 1].device != ctx->device) return true;
    return false;
}

// Resolve a segment's kernel (patched image when available) and its per-entry grid.
static int setup_seg(sw_ctx *ctx, const Job &J, Seg &G, int P, int NS, bool tail, int cp, const int *cg)
{
    const Variant &V = *G.V;
    G.BH = V.alpha * 32 * V.nw;
    // special rows off the strip bottoms (k not a multiple of alpha, or a segment
    // starting off a multiple of alpha): the GEN instantiation
    const bool gen = G.use16 && J.local && J.k > 0 && (J.k % V.alpha != 0 || G.row_base % V.alpha != 0);
    G.fn = G.use16 ? (J.local ? (gen ? V.packed_gen_fn : V.packed_fn) : V.packed_global_fn)
                   : J.wide ? (J.local ? V.local_wide_fn : V.global_wide_fn) : (J.local ? V.local_fn : V.global_fn);
    if (!G.fn) {
        snprintf(ctx->errbuf, sizeof(ctx->errbuf), "no kernel for geometry alpha %d x %d warps (gen %d)", V.alpha, V.nw, gen ? 1 : 0);
        return SW_EINVAL;
    }
    G.smem = G.use16 ? V.smem16 : V.smem;
    G.patched = false;
    if (const void *pf = patched_kernel(ctx, V, J.ge, J.go + J.ge, G.use16 ? (J.local ? (gen ? 4 : 0) : 3) : J.local ? 1 : 2)) {
        G.fn = pf;
        G.patched = true;
    }
    // the tail launch asks for enough shared memory to hold one CTA per SM:
    // its CTAs take the SMs the main launch frees one by one
    if (tail) G.smem = std::max<size_t>(G.smem, (size_t)TAIL_SMEM);
    G.block = V.nw * 32 + (G.use16 ? V.io_warps : 1) * 32;
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, G.fn, G.block, G.smem);
    if (per_sm < 1) per_sm = 1;
    for (int d = 0; d < P; d++) {
        // every CTA of every stripe / entry must be co-resident (they wait on each other)
        const int cap = std::max(1, per_sm * ctx->num_sms / (NS * (P > 1 ? ctx->share[d] : 1)));
        const int bands_d = (G.nb - cg[d] + cp - 1) / cp;  // bands b = t cp + cg[d] of this entry
        int g = std::max(1, std::min(bands_d, cap));
        if (const char *e = getenv("SWB_GRID")) g = std::max(1, std::min(g, atoi(e) / NS));
        if (ctx->grid_cap > 0) g = std::max(1, std::min(g, ctx->grid_cap / NS));
        G.grid[d] = g * NS;
    }
    return SW_OK;
}

// Tail segment: when a multi-wave fill leaves a partial last
// wave (C4: 1221 bands of 8192 rows on 148 CTAs, the ninth wave a quarter
// full), run the rows after the last full wave as a second launch of a
// geometry with shorter bands, so they spread over every SM instead of a
// quarter of them.  Returns the tail geometry and the main launch's band count,
// or nullptr.  Automatic choice by the band-pipeline model; sw_set_tail forces.
static const Variant *choose_tail(sw_ctx *ctx, const Job &J, const Seg &S0, int *nb1_out)
{
    if (ctx->tail_mode == 0 || (ctx->tail_mode < 0 && ctx->variant_override >= 0)) return nullptr;
    const int P = S0.grid[0];
    const int nb = S0.nb;
    const int nb1 = (nb / P) * P;
    if (nb <= P || nb1 == nb) return nullptr;  // one wave, or whole waves only
    const long long m2 = J.m - (long long)nb1 * S0.BH;
    const long long n = std::max<long long>(J.n, 1);
    const Variant &V0 = *S0.V;
    const int vidx0 = (int)(&V0 - &variant_for(0));
    if (ctx->tail_mode > 0) {
        const Variant &Vt = variant_for(ctx->tail_mode - 1);
        if (!packed_qualifies(ctx, J, Vt) || Vt.alpha * 32 * Vt.nw >= S0.BH) return nullptr;
        if (J.k > 0 && ((long long)nb1 * S0.BH) % Vt.alpha != 0 && !Vt.packed_gen_fn) return nullptr;
        *nb1_out = nb1;
        return &Vt;
    }
    double cps0 = 0;
    for (int c = 0; c < NCANDS; c++)
        if (kCands[c].variant == vidx0 && kCands[c].packed) cps0 = kCands[c].cps_full;
    if (cps0 <= 0) return nullptr;
    const long long lag0 = (2ll * V0.nw + 2) * V0.w;
    const double t_no = model_fill_time(nb, P, n, lag0, cps0);
    double best = 0.97 * t_no;
    const Variant *pick = nullptr;
    for (const Candidate &C : kTailCands) {
        const Variant &Vt = variant_for(C.variant);
        const long long bh = (long long)Vt.alpha * 32 * Vt.nw;
        if (bh >= S0.BH || !packed_qualifies(ctx, J, Vt)) continue;
        if (J.k > 0 && ((long long)nb1 * S0.BH) % Vt.alpha != 0 && !Vt.packed_gen_fn) continue;
        const long long nb2 = (m2 + bh - 1) / bh;
        if (nb2 > ctx->num_sms) continue;  // the tail must fit in one wave of one CTA per SM
        const long long lagt = (2ll * Vt.nw + 2) * Vt.w;
        const double t = model_fill_time(nb1, P, n, lag0, cps0) + ((double)n + (double)(nb2 - 1) * lagt) / C.cps_solo;
        if (t < best) {
            best = t;
            pick = &Vt;
        }
    }
    if (pick) *nb1_out = nb1;
    return pick;
}

static int run_job(sw_ctx *ctx, const Job &J0, cudaStream_t user_stream, int4 *res)
{
    Job J = J0;
    J.wide = std::abs((long long)J.ma + J.go + J.ge) > 127 || std::abs((long long)J.mi + J.go + J.ge) > 127;
    const auto h0 = std::chrono::steady_clock::now();
    if (J.local) ctx->s1.valid = false;
    auto hnow = [&]() { return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - h0).count(); };
    // band-cyclic multi-GPU Stage 1: entry d runs bands d, d + P, ...
    // or column stripes, one per entry (mstr), with the (t, E) border column
    // stored into the next entry's receive area
    const bool rcyc = J.rank_cyc;
    const bool multi = J.local && !J.rank_mode && !rcyc && J.nv == 1 && ctx->ndev > 1;
    const bool cyc = multi && ctx->cyclic;
    const bool mstr = multi && !ctx->cyclic;
    const int P = multi ? ctx->ndev : 1;
    const bool cross = (multi && distinct_devices(ctx)) || rcyc;
    // the band-cyclic step and index of each entry (1, 0: every band)
    const int cp = cyc ? P : rcyc ? J.cyc_world : 1;
    int cg[MAX_DEV] = {};
    for (int d = 0; d < P; d++) cg[d] = cyc ? d : rcyc ? J.cyc_rank : 0;
    const int NS = (J.rank_mode || multi) ? 1 : J.nv;  // column stripes of one launch
    const int NU = multi ? P : NS;                     // units: (entry, stripe) buffer sets
    Seg seg[2];
    int nseg = 1;
    seg[0].V = &choose_variant(ctx, J, &seg[0].use16, cp);
    const Variant &V = *seg[0].V;
    const int W = V.w;
    const int m = (int)J.m, n = (int)J.n;
    seg[0].BH = V.alpha * 32 * V.nw;
    seg[0].nb = (m + seg[0].BH - 1) / seg[0].BH;
    int rc;
    if ((rc = setup_seg(ctx, J, seg[0], P, NS, false, cp, cg))) return rc;
    // the last partial wave of a multi-wave fill as a second launch with a
    // smaller band height
    if (cp == 1 && !multi && NS == 1 && !J.rank_mode && J.local && seg[0].use16) {
        int nb1 = 0;
        const Variant *Vt = choose_tail(ctx, J, seg[0], &nb1);
        if (Vt) {
            seg[1].V = Vt;
            seg[1].use16 = true;
            seg[1].row_base = nb1 * seg[0].BH;
            seg[1].band_base = nb1;
            seg[1].BH = Vt->alpha * 32 * Vt->nw;
            seg[1].nb = (m - seg[1].row_base + seg[1].BH - 1) / seg[1].BH;
            seg[0].nb = nb1;
            if ((rc = setup_seg(ctx, J, seg[0], P, NS, false, cp, cg))) return rc;
            if ((rc = setup_seg(ctx, J, seg[1], P, NS, true, cp, cg))) return rc;
            nseg = 2;
        }
    }
    const int nb_total = seg[0].nb + (nseg > 1 ? seg[1].nb : 0);
    const double h_choose = hnow();
    const long long wa = (J.m + 15) / 16 + 2, wb = (J.n + 15) / 16 + 2;

    // stripe geometry (units of the band-cyclic mode all span [0, n))
    long long col0[MAX_STRIPES], wid[MAX_STRIPES];
    int udev[MAX_STRIPES];  // device entry of each unit
    for (int u = 0; u < NU; u++) {
        udev[u] = multi ? u : 0;
        if (J.rank_mode) { col0[u] = J.c_lo; wid[u] = J.c_hi - J.c_lo; }
        else if (cyc || rcyc) { col0[u] = 0; wid[u] = n; }
        else { col0[u] = (long long)n * u / NU; wid[u] = (long long)n * (u + 1) / NU - col0[u]; }
        if (wid[u] <= 0) {
            snprintf(ctx->errbuf, sizeof(ctx->errbuf), "stripe %d is empty (n=%d, stripes=%d)", u, n, NS);
            return SW_EINVAL;
        }
    }
    auto devof = [&](int d) { return d == 0 ? ctx->device : ctx->peer[d - 1].device; };
    auto setdev = [&](int d) { return cudaSetDevice(devof(d)); };

    // ---- per-entry buffers: codes (entry 0 encodes; peers on other GPUs get a copy), misc, slots
    int grid_sum[MAX_DEV] = {};
    for (int d = 0; d < P; d++)
        for (int g = 0; g < nseg; g++) grid_sum[d] += seg[g].grid[d];
    for (int d = 0; d < P; d++) {
        DevView D = dview(ctx, d);
        CK(setdev(d));
        const bool own_codes = d == 0 || devof(d) != ctx->device;
        if (own_codes) {
            if ((rc = grow(ctx, *D.a2, wa * 4))) return rc;
            if ((rc = grow(ctx, *D.b2, wb * 4))) return rc;
        }
        if ((rc = grow(ctx, *D.misc, 256))) return rc;
        if ((rc = grow(ctx, *D.slots, (size_t)grid_sum[d] * sizeof(int4)))) return rc;
    }
    CK(setdev(0));
    if (J.match && (rc = grow(ctx, ctx->capbuf, ((size_t)nb_total * seg[0].BH + 2) * sizeof(int2)))) return rc;
    const size_t border_rows = (size_t)seg[0].nb * seg[0].BH + 2;
    const size_t border_flags = (size_t)seg[0].nb * V.nw + 1;
    int NT[MAX_STRIPES];
    for (int u = 0; u < NU; u++) {
        CK(setdev(udev[u]));
        if (ctx->unit_dev[u] != devof(udev[u])) {
            // the unit moved to another device (multi-device vs single-device calls)
            for (DevBuf *b : {&ctx->rowb[u], &ctx->progress[u], &ctx->sp[u]}) {
                if (b->p) cudaFree(b->p);
                *b = DevBuf{};
            }
            if (ctx->vrecv[u].base) cudaFree(ctx->vrecv[u].base);
            ctx->vrecv[u] = RecvArea{};
            ctx->unit_dev[u] = devof(udev[u]);
        }
        const int npad = (int)((wid[u] + W - 1) / W) * W;
        NT[u] = npad / W + (seg[0].use16 ? 1 : V.skew_tiles);
        if (rcyc) {
            // the exported / imported areas hold the row border and the band progress
            if (!ctx->cin || !ctx->cout || ctx->cin_cols < (size_t)(NT[u] * W + 2 * W) ||
                ctx->cout_cols < (size_t)(NT[u] * W + 2 * W) || ctx->cin_bands < (size_t)nb_total + 2 ||
                ctx->cout_bands < (size_t)nb_total + 2) {
                snprintf(ctx->errbuf, sizeof(ctx->errbuf), "band-cyclic areas missing or too small (sw_cyclic_export / connect)");
                return SW_EINVAL;
            }
            continue;
        }
        if ((rc = grow(ctx, ctx->rowb[u], (size_t)(NT[u] * W + 2 * W) * sizeof(int2)))) return rc;
        const size_t pbytes = (size_t)(nb_total + 2) * sizeof(unsigned long long);
        if (ctx->progress[u].cap < pbytes || !ctx->progress[u].p) {
            if ((rc = grow(ctx, ctx->progress[u], pbytes))) return rc;
            CK(cudaMemset(ctx->progress[u].p, 0, ctx->progress[u].cap));  // tags of earlier calls are 0 here
        }
        if (!J.rank_mode && !cyc && u > 0)
            if ((rc = grow_recv(ctx, ctx->vrecv[u], border_rows, border_flags))) return rc;
    }
    CK(setdev(0));
    if (J.rank_mode) {
        if (J.c_lo > 0 && (!ctx->recv.base || ctx->recv.rows < border_rows || ctx->recv.flags < border_flags)) {
            snprintf(ctx->errbuf, sizeof(ctx->errbuf), "stripe receive area missing or too small (sw_stripe_export)");
            return SW_EINVAL;
        }
        if (J.c_hi < n && (!ctx->right_base || ctx->right_rows < border_rows)) {
            snprintf(ctx->errbuf, sizeof(ctx->errbuf), "right neighbour not connected (sw_stripe_connect)");
            return SW_EINVAL;
        }
    }

    // ---- special rows (a6): a ring of R slots per unit in HBM, streamed to the
    // host as bands complete; R = every row when they fit the device budget,
    // else as many as fit (at least one band's rows), with back-pressure
    // (sp_admit) and a host store for Stage 2 (the paper's SRA).
    const long long nsp = (J.local && J.k > 0) ? J.m / J.k : 0;
    int ld[MAX_STRIPES];
    long long stride[MAX_STRIPES];
    size_t slot_bytes = 0;  // bytes of one ring slot on the busiest device
    for (int u = 0; u < NU; u++) {
        ld[u] = (int)((wid[u] + 31) / 32) * 32;
        stride[u] = 2ll * ld[u];
        if (multi) slot_bytes = std::max(slot_bytes, (size_t)stride[u] * sizeof(int));
        else slot_bytes += (size_t)stride[u] * sizeof(int);
    }
    long long R = nsp;
    bool store = false;
    if (nsp > 0) {
        long long rpb = 1;  // most special rows one band can hold
        for (int g = 0; g < nseg; g++) rpb = std::max<long long>(rpb, (seg[g].BH + J.k - 1) / J.k + 1);
        const long long R_min = std::min<long long>(nsp, rpb);
        bool grows = false;
        size_t have = 0;
        for (int u = 0; u < NU; u++) {
            have += ctx->sp[u].cap;
            grows |= ctx->sp[u].cap < (size_t)nsp * stride[u] * sizeof(int);
        }
        if (ctx->sp_budget > 0 || grows) {
            // only when the buffers must grow: cudaMemGetInfo can take
            // milliseconds (it stalled repeated calls by up to 19 ms)
            size_t freeb = 0, totb = 0;
            if (grows) cudaMemGetInfo(&freeb, &totb);
            const double avail = (double)freeb + (double)(multi ? have / std::max(1, P) : have);
            double budget = grows ? 0.8 * avail : 1e30;
            if (ctx->sp_budget > 0) budget = std::min(budget, (double)ctx->sp_budget);
            if ((double)nsp * slot_bytes > budget) {
                R = std::max<long long>(R_min, (long long)(budget / (double)slot_bytes));
                if (grows && (double)R * slot_bytes > 0.95 * avail) {
                    snprintf(ctx->errbuf, sizeof(ctx->errbuf), "special-row ring of %lld rows needs %zu bytes on the device",
                             R, (size_t)R * slot_bytes);
                    return SW_ENOMEM;
                }
            }
        } else if (ctx->sp_budget == 0) {
            R = nsp;
        }
        store = (R < nsp || multi) && NS == 1 && !J.rank_mode && !rcyc;
        if (store) {
            // the host store (the SRA) may take at most half the physical memory:
            // a larger one would page the host out (Stage 2 then refuses: SW_EINVAL)
            const double phys = (double)sysconf(_SC_PHYS_PAGES) * (double)sysconf(_SC_PAGE_SIZE);
            if ((double)nsp * 8.0 * (double)n > 0.5 * phys) store = false;
        }
        for (int u = 0; u < NU; u++) {
            CK(setdev(udev[u]));
            if ((rc = grow(ctx, ctx->sp[u], (size_t)R * stride[u] * sizeof(int)))) return rc;
            if ((rc = grow_host(ctx, ctx->flags[u], nsp * sizeof(unsigned int), true))) return rc;
            memset(ctx->flags[u].p, 0, nsp * sizeof(unsigned int));
            if ((rc = grow_host(ctx, ctx->colp[u], (size_t)nb_total * sizeof(unsigned int), true))) return rc;
            memset(ctx->colp[u].p, 0, (size_t)nb_total * sizeof(unsigned int));
        }
        CK(setdev(0));
        // staging window: every special row when they fit in ~1 GiB of pinned
        // memory (a one-wave matrix completes all its rows together), else as
        // many as fit (at least 2)
        const size_t row_bytes = (size_t)2 * (n + 64) * sizeof(int32_t);
        ctx->nstage = (int)std::max<size_t>(2, std::min<size_t>((size_t)nsp, ((size_t)1 << 30) / row_bytes));
        if ((rc = grow_host(ctx, ctx->stage, row_bytes * ctx->nstage, false))) return rc;
        for (int d = 0; d < P; d++) {
            DevView D = dview(ctx, d);
            CK(setdev(d));
            while ((int)D.ev_row->size() < ctx->nstage) {
                cudaEvent_t ev;
                CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
                D.ev_row->push_back(ev);
            }
        }
        CK(setdev(0));
        if (store) {
            ctx->host_rows.resize((size_t)nsp);
            for (auto &r : ctx->host_rows) r.clear();
        }
    }
    *(volatile unsigned long long *)ctx->released.p = 0ull;
    unsigned long long *d_released = nullptr;

    // ---- launches.  With a caller stream, every kernel of entry 0 is launched
    // on it (so the caller's CUDA events bracket them); otherwise on the
    // library stream.  The tail segment runs on the aux stream, the main
    // stream waits for it.
    const double h_alloc = hnow();
    cudaStream_t st = user_stream ? user_stream : ctx->stream;
    char *misc0 = (char *)ctx->misc.p;
    int *d_err = (int *)(misc0 + 0);
    // progress tags: the ranks' agreed epoch (the next rank's area holds tags
    // of earlier agreed epochs only), else this context's own counter
    const int pepoch = rcyc ? J.epoch : ++ctx->pepoch;
    if (rcyc) ctx->pepoch = std::max(ctx->pepoch, J.epoch);
    CK(cudaEventRecord(ctx->ev[0], st));
    for (int d = 0; d < P; d++) {
        DevView D = dview(ctx, d);
        cudaStream_t sd = d == 0 ? st : D.stream;
        CK(setdev(d));
        char *misc = (char *)D.misc->p;
        CK(cudaMemsetAsync(misc, 0, 16, sd));
        CK(cudaMemsetAsync(misc + 12, 0x7f, 4, sd));  // hit_band
        CK(cudaMemsetAsync(misc + 16, 0xff, 8, sd));  // hit_key
        CK(cudaMemsetAsync(misc + 24, 0, 8, sd));     // replays
        CK(cudaMemsetAsync(misc + 64, 0, 2 * MAX_STRIPES * sizeof(int), sd));  // tickets (2 segments)
    }
    CK(setdev(0));
    {
        const long long words = wa + wb;
        const int tpb = 256;
        sw_encode_kernel<<<(unsigned)((words + tpb - 1) / tpb), tpb, 0, st>>>(
            J.dA, J.m, J.revA, (uint32_t *)ctx->a2.p, wa, J.dB, J.n, J.revB, (uint32_t *)ctx->b2.p, wb, d_err);
        CK(cudaGetLastError());
    }
    CK(cudaEventRecord(ctx->ev[1], st));
    const double h_encode = hnow();

    auto fill_args = [&](int d, const Seg &G) -> FillArgs {
        DevView D = dview(ctx, d);
        char *misc = (char *)D.misc->p;
        const bool own_codes = d == 0 || devof(d) != ctx->device;
        FillArgs a{};
        a.m = m;
        a.n = n;
        a.nb = G.nb;
        a.row_base = G.row_base;
        a.band_base = G.band_base;
        a.cyc_p = cp;
        a.cyc_g = cg[d];
        a.cross = cross ? 1 : 0;
        a.go = J.go;
        a.ge = J.ge;
        a.gf = J.go + J.ge;
        a.one = 1;
        a.pm_gf = J.ma + a.gf;
        a.pn_gf = J.mi + a.gf;
        for (int x = 0; x < 4; x++) {
            uint32_t w = 0;
            for (int y = 0; y < 4; y++) {
                const int v = (x == y ? J.ma : J.mi) + a.gf;
                w |= (uint32_t)(uint8_t)(int8_t)v << (8 * y);
            }
            a.prof[x] = w;
        }
        a.A2 = (const uint32_t *)(own_codes ? D.a2->p : ctx->a2.p);
        a.B2 = (const uint32_t *)(own_codes ? D.b2->p : ctx->b2.p);
        a.err = d_err;  // entry 0's: an alphabet error stops every entry
        a.k = (int)(nsp > 0 ? J.k : 0);
        a.sp_slots = (int)std::max<long long>(1, R);
        a.sp_released = (R < nsp && !getenv("SWB_NO_ADMIT")) ? d_released : nullptr;
        a.admit_ns = getenv("SWB_ADMIT_NS") ? (unsigned)atoi(getenv("SWB_ADMIT_NS")) : 2000u;
        a.gbest = (int *)(misc + 8);
        a.goal = J.goal;
        a.hit_w = J.hit_w;
        a.anchor_gap = J.anchor_gap ? 1 : 0;
        a.match = J.match ? 1 : 0;
        a.mjc = (int)J.mjc;
        a.mH = J.mH;
        a.mF = J.mF;
        a.hit_key = (unsigned long long *)(misc + 16);
        a.hit_band = (int *)(misc + 12);
        a.replays = (unsigned long long *)(misc + 24);
        a.epoch = J.epoch;
        a.pepoch = pepoch;
        a.timeout_ns = ctx->timeout_ns;
        a.nstripes = NS;
        a.force_slow = 0;
        a.dbg = nullptr;
        return a;
    };
    auto fill_stripes = [&](FillArgs &a, int d, int segi) -> int {
        const Seg &G = seg[segi];
        for (int s = 0; s < NS; s++) {
            const int u = multi ? d : s;
            StripeArgs &S = a.st[s];
            S.col0 = (int)col0[u];
            S.w = (int)wid[u];
            S.ncols_pad = (int)((wid[u] + W - 1) / W) * W;
            S.NT = NT[u];
            const int un = cyc ? (u + 1) % P : u;  // the unit that runs the next band
            S.rowb_in = (const int2 *)ctx->rowb[u].p;
            S.rowb_out = (int2 *)ctx->rowb[un].p;
            S.prog_in = (const unsigned long long *)ctx->progress[u].p;
            S.prog_out = (unsigned long long *)ctx->progress[un].p;
            if (rcyc) {  // this rank's incoming area, and the next rank's over CUDA IPC / NVLink
                S.rowb_in = (const int2 *)ctx->cin;
                S.prog_in = (const unsigned long long *)((const char *)ctx->cin + ctx->cin_cols * sizeof(int2));
                S.rowb_out = (int2 *)ctx->cout;
                S.prog_out = (unsigned long long *)((char *)ctx->cout + ctx->cout_cols * sizeof(int2));
            }
            S.ticket = (int *)((char *)dview(ctx, d).misc->p + 64) + segi * MAX_STRIPES + s;
            S.sp = nsp > 0 ? (int *)ctx->sp[u].p : nullptr;
            S.sp_stride = stride[u];
            S.sp_ld = ld[u];
            unsigned int *fd = nullptr, *cp = nullptr;
            if (nsp > 0) {
                CK(cudaHostGetDevicePointer((void **)&fd, ctx->flags[u].p, 0));
                CK(cudaHostGetDevicePointer((void **)&cp, ctx->colp[u].p, 0));
            }
            S.row_done = fd;
            S.colp = cp;
            S.lb = nullptr; S.lready = nullptr; S.rb = nullptr; S.rready = nullptr;
            if (mstr) {
                S.lb = u > 0 ? ctx->vrecv[u].lb() : nullptr;
                S.lready = u > 0 ? ctx->vrecv[u].lready() : nullptr;
                S.rb = u + 1 < P ? ctx->vrecv[u + 1].lb() : nullptr;
                S.rready = u + 1 < P ? ctx->vrecv[u + 1].lready() : nullptr;
            } else if (J.rank_mode) {
                S.lb = J.c_lo > 0 ? ctx->recv.lb() : nullptr;
                S.lready = J.c_lo > 0 ? ctx->recv.lready() : nullptr;
                RecvArea right;
                right.base = ctx->right_base;
                right.rows = ctx->right_rows;
                S.rb = J.c_hi < n ? right.lb() : nullptr;
                S.rready = J.c_hi < n ? right.lready() : nullptr;
            } else if (!cyc) {
                S.lb = s > 0 ? ctx->vrecv[s].lb() : nullptr;
                S.lready = s > 0 ? ctx->vrecv[s].lready() : nullptr;
                S.rb = s + 1 < NS ? ctx->vrecv[s + 1].lb() : nullptr;
                S.rready = s + 1 < NS ? ctx->vrecv[s + 1].lready() : nullptr;
                if (J.match) {  // Stage 2: capture the last column for the band-end matching
                    S.rb = (int2 *)ctx->capbuf.p;
                    S.rready = nullptr;
                }
            }
        }
        (void)G;
        return SW_OK;
    };
    auto launch = [&](const Seg &G, int d, FillArgs &a, cudaStream_t sd, int slot_off) -> int {
        a.slots = (int4 *)dview(ctx, d).slots->p + slot_off;
        void *args[] = {&a};
        const cudaError_t le = cudaLaunchKernel(G.fn, dim3(G.grid[d]), dim3(G.block), args, G.smem, sd);
        if (le != cudaSuccess) {
            cudaGetLastError();  // not sticky: do not fail the context's next call
            return cuda_fail(ctx, le, "cudaLaunchKernel(fill)");
        }
        return SW_OK;
    };
    for (int d = 0; d < P; d++) {
        DevView D = dview(ctx, d);
        cudaStream_t sd = d == 0 ? st : D.stream;
        CK(setdev(d));
        if (nsp > 0 && R < nsp) CK(cudaHostGetDevicePointer((void **)&d_released, ctx->released.p, 0));
        if (d > 0) {
            CK(cudaStreamWaitEvent(sd, ctx->ev[1], 0));
            if (devof(d) != ctx->device) {
                CK(cudaMemcpyPeerAsync(D.a2->p, devof(d), ctx->a2.p, ctx->device, wa * 4, sd));
                CK(cudaMemcpyPeerAsync(D.b2->p, devof(d), ctx->b2.p, ctx->device, wb * 4, sd));
            }
        }
        FillArgs a = fill_args(d, seg[0]);
        if ((rc = fill_stripes(a, d, 0))) return rc;
        if (d == 0 && getenv("SWB_DEBUG_TIMES")) {
            if ((rc = grow(ctx, ctx->dbg, (size_t)nb_total * 80 * sizeof(unsigned long long)))) return rc;
            CK(cudaMemsetAsync(ctx->dbg.p, 0, (size_t)nb_total * 80 * sizeof(unsigned long long), st));
            a.dbg = (unsigned long long *)ctx->dbg.p;
            ctx->dbg_n = nb_total;
        }
        if ((rc = launch(seg[0], d, a, sd, 0))) return rc;
        if (nseg > 1) {
            FillArgs at = fill_args(d, seg[1]);
            if ((rc = fill_stripes(at, d, 1))) return rc;
            at.dbg = a.dbg;
            CK(cudaStreamWaitEvent(ctx->aux, ctx->ev[1], 0));
            if ((rc = launch(seg[1], d, at, ctx->aux, seg[0].grid[d]))) return rc;
            CK(cudaEventRecord(ctx->ev_aux[0], ctx->aux));
            CK(cudaStreamWaitEvent(st, ctx->ev_aux[0], 0));
        }
        if (d > 0) CK(cudaEventRecord(D.ev[2], sd));
    }
    CK(setdev(0));
    for (int d = 1; d < P; d++) CK(cudaStreamWaitEvent(st, dview(ctx, d).ev[2], 0));
    CK(cudaEventRecord(ctx->ev[2], st));
    auto enqueue_results = [&]() -> int {
        for (int d = 0; d < P; d++) {
            DevView D = dview(ctx, d);
            cudaStream_t sd = d == 0 ? st : D.stream;
            CK(setdev(d));
            char *misc = (char *)D.misc->p;
            sw_reduce_kernel<<<1, 256, 0, sd>>>((const int4 *)D.slots->p, grid_sum[d], J.local ? 1 : 0,
                                                (const unsigned long long *)(misc + 16), J.goal, (int4 *)(misc + 32));
            CK(cudaGetLastError());
            CK(cudaMemcpyAsync(D.res_h, misc + 32, sizeof(int4), cudaMemcpyDeviceToHost, sd));
            CK(cudaMemcpyAsync(D.res_h + 1, d_err, sizeof(int), cudaMemcpyDeviceToHost, sd));
            CK(cudaMemcpyAsync(D.res_h + 2, misc + 24, sizeof(unsigned long long), cudaMemcpyDeviceToHost, sd));
            if (d > 0) CK(cudaEventRecord(D.ev[3], sd));
        }
        CK(setdev(0));
        CK(cudaEventRecord(ctx->ev[3], st));
        return SW_OK;
    };
    // The result copies are enqueued after the special-row loop: a device-to-host
    // copy queued behind the running fill on its stream held back every other
    // stream's device-to-host copies until the fill ended (measured: special rows
    // reached the host only after the fill, and a ring that waits on the host
    // for its slots never drained; profiles/r02_copy_order.txt).

    // ---- stream special rows to the sink (and the host store) in ascending
    // order while the fill runs.  A staged row is copied in column chunks as
    // its band publishes final columns (colp), and completed once every unit
    // holding a slice of it has published the row (row_done); the sink then
    // runs on it in row order, and its ring slot is released.
    int sink_rc = 0;
    long long bytes = 0;
    const int64_t nrow_out = J.rank_mode ? wid[0] : n;
    const int64_t sld = (NU == 1 || cyc) ? ld[0] : nrow_out + 32;  // H at [0, sld), F at [sld, 2 sld)
    const int nstage = nsp > 0 ? ctx->nstage : 0;
    const int64_t CHUNK = 65536;  // columns per partial copy (512 KiB of H + F)
    std::vector<int64_t> copied((size_t)nstage * NU, 0);
    std::vector<char> sealed(nstage, 0);
    std::vector<int> sealdev(nstage, 0);
    const bool dbg_host = nsp > 0 && getenv("SWB_DEBUG_HOST") != nullptr;
    double h_fill = -1, h_sink_max = 0;
    long long n_copies = 0;
    // global band of DP row `row` (1-based) and the unit that ran it
    auto band_of = [&](long long row) -> int {
        const long long r0 = row - 1;
        if (nseg > 1 && r0 >= seg[1].row_base) return seg[1].band_base + (int)((r0 - seg[1].row_base) / seg[1].BH);
        return (int)(r0 / seg[0].BH);
    };
    auto unit_lo = [&](long long q) { return cyc ? band_of((q + 1) * J.k) % P : 0; };
    // rows of this process (band-cyclic ranks: only the rows of this rank's bands)
    auto mine = [&](long long q) { return !rcyc || band_of((q + 1) * J.k) % cp == J.cyc_rank; };
    auto unit_hi = [&](long long q) { return cyc ? unit_lo(q) + 1 : NU; };
    auto row_ready = [&](long long q) -> bool {
        for (int u = unit_lo(q); u < unit_hi(q); u++)
            if (((volatile unsigned int *)ctx->flags[u].p)[q] == 0) return false;
        return true;
    };
    auto release_all = [&]() { *(volatile unsigned long long *)ctx->released.p = ~0ull >> 1; };
    auto fill_running = [&]() -> cudaError_t {
        for (int d = P - 1; d >= 0; d--) {
            const cudaError_t e = cudaEventQuery(dview(ctx, d).ev[d == 0 ? 2 : 2]);
            if (e != cudaSuccess) return e;
        }
        return cudaSuccess;
    };
    // last DP row (1-based, inclusive) of global band G
    auto band_end = [&](int G) -> long long {
        long long e = (nseg > 1 && G >= seg[1].band_base)
                          ? (long long)seg[1].row_base + (long long)(G - seg[1].band_base + 1) * seg[1].BH
                          : (long long)(G + 1) * seg[0].BH;
        return std::min<long long>(e, J.m);
    };
    // one side stream per row, so that one event seals it: the owning entry's
    // (band-cyclic), else entry 0's (column slices of other entries are read over the peer mapping)
    auto copy_dev = [&](long long q) { return cyc ? band_of((q + 1) * J.k) % P : 0; };
    // copy what is final of the staged rows [q0, q1) of one band (ready: the band has ended)
    const int copy_mode = getenv("SWB_COPY_MODE") ? atoi(getenv("SWB_COPY_MODE")) : 0;
    cudaStream_t dbg_stream = nullptr;
    if (copy_mode == 3) cudaStreamCreateWithFlags(&dbg_stream, cudaStreamNonBlocking);
    auto pump_band = [&](long long q0, long long q1, int band, bool ready, bool &moved) -> int {
        const int d = copy_dev(q0);
        DevView D = dview(ctx, d);
        if (copy_mode == 2) D.side = ctx->aux;
        if (copy_mode == 3) D.side = dbg_stream;
        bool devset = false;
        int64_t av[MAX_STRIPES];
        const int ulo = unit_lo(q0), uhi = unit_hi(q0);
        for (int u = ulo; u < uhi; u++)
            av[u] = ready ? wid[u] : std::min<int64_t>(wid[u], ((volatile unsigned int *)ctx->colp[u].p)[band]);
        for (long long q = q0; q < q1; q++) {
            const int slot = (int)(q % nstage);
            if (sealed[slot]) continue;
            bool all = true;
            int32_t *dst = (int32_t *)ctx->stage.p + (size_t)slot * 2 * sld;
            for (int u = ulo; u < uhi; u++) {
                int64_t &c = copied[(size_t)slot * NU + u];
                if (av[u] > c && (ready || av[u] - c >= CHUNK)) {
                    if (!devset) {
                        CK(setdev(d));
                        devset = true;
                    }
                    const int32_t *src = (const int32_t *)ctx->sp[u].p + (q % R) * stride[u] + c;
                    const int64_t off = (NU == 1 || J.rank_mode || cyc) ? 0 : col0[u];
                    if (copy_mode == 1) {
                        CK(cudaMemcpyAsync(dst + off + c, src, (size_t)(av[u] - c) * 4, cudaMemcpyDeviceToHost, D.side));
                        CK(cudaMemcpyAsync(dst + sld + off + c, src + ld[u], (size_t)(av[u] - c) * 4, cudaMemcpyDeviceToHost, D.side));
                    } else {
                        CK(cudaMemcpy2DAsync(dst + off + c, (size_t)sld * 4, src, (size_t)ld[u] * 4, (size_t)(av[u] - c) * 4, 2,
                                             cudaMemcpyDeviceToHost, D.side));
                    }
                    n_copies++;
                    c = av[u];
                    moved = true;
                }
                if (c < wid[u]) all = false;
            }
            if (ready && all) {
                if (!devset) {
                    CK(setdev(d));
                    devset = true;
                }
                CK(cudaEventRecord((*D.ev_row)[slot], D.side));
                sealed[slot] = 1;
                sealdev[slot] = d;
                moved = true;
            }
        }
        return SW_OK;
    };
    // on an error in this loop the kernels may wait on the ring: release it
    // and let them finish before returning
    auto bail = [&](int code) -> int {
        release_all();
        for (int d = 0; d < P; d++) {
            setdev(d);
            cudaStreamSynchronize(d == 0 ? st : dview(ctx, d).stream);
            cudaStreamSynchronize(dview(ctx, d).side);
        }
        setdev(0);
        return code;
    };
    auto release = [&](long long upto) { *(volatile unsigned long long *)ctx->released.p = (unsigned long long)upto; };
    long long done = (J.sink || store) ? 0 : nsp;  // no sink and resident rows (sw_align): nothing to copy
    while (done < nsp) {
        bool progress = false;
        if (dbg_host && h_fill < 0 && fill_running() == cudaSuccess) h_fill = hnow();
        // 1) copy what is final of the staged window, one band at a time (two
        //    mapped-flag reads per band, not per row)
        const long long hi = std::min<long long>(nsp, done + nstage);
        for (long long q = done; q < hi;) {
            const int band = band_of((q + 1) * J.k);
            const long long q1 = std::min<long long>(hi, std::max<long long>(q + 1, band_end(band) / J.k));
            if (mine(q) && (rc = pump_band(q, q1, band, row_ready(q), progress))) return bail(rc);
            q = q1;
        }
        // 2) hand every completed row to the sink in order and free its ring slot
        while (done < nsp) {
            if (!mine(done)) {  // another rank's row: it never occupies this rank's ring
                release(++done);
                progress = true;
                continue;
            }
            const int slot = (int)(done % nstage);
            if (!sealed[slot]) break;
            setdev(sealdev[slot]);
            const cudaError_t qe = cudaEventQuery((*dview(ctx, sealdev[slot]).ev_row)[slot]);
            if (qe == cudaErrorNotReady) break;
            if (qe != cudaSuccess) return bail(cuda_fail(ctx, qe, "special-row copy"));
            bytes += 8ll * nrow_out;
            int32_t *row = (int32_t *)ctx->stage.p + (size_t)slot * 2 * sld;
            if (store) {
                std::vector<int32_t> &hr = ctx->host_rows[(size_t)done];
                try {
                    hr.resize((size_t)2 * n);
                    memcpy(hr.data(), row, (size_t)n * 4);
                    memcpy(hr.data() + n, row + sld, (size_t)n * 4);
                } catch (...) {
                    store = false;  // no host memory for the SRA: Stage 2 will refuse
                    ctx->host_rows.clear();
                }
            }
            const double t0 = dbg_host ? hnow() : 0;
            if (dbg_host && (done == 0 || done + 1 == nsp || done % 256 == 0))
                fprintf(stderr, "[swb host] row %lld to the sink at %.3f ms (fill %s)\n", done, t0,
                        fill_running() == cudaSuccess ? "done" : "running");
            if (J.sink && J.sink(J.user, (done + 1) * J.k, row, row + sld, nrow_out)) sink_rc = SW_EABORTED;
            if (dbg_host) h_sink_max = std::max(h_sink_max, hnow() - t0);
            sealed[slot] = 0;
            for (int u = 0; u < NU; u++) copied[(size_t)slot * NU + u] = 0;
            release(++done);  // the row's ring slot is free: the back-pressure counter
            progress = true;
            if (sink_rc) break;
        }
        if (sink_rc) break;
        if (!progress && done < nsp) {
            // nothing ready: make sure the fill is still running
            const int slot = (int)(done % nstage);
            const cudaError_t fe = fill_running();
            if (fe == cudaSuccess && !sealed[slot] && !row_ready(done)) {
                bail(0);
                if (ctx->res_h[1].x == 1) return SW_EALPHABET;
                snprintf(ctx->errbuf, sizeof(ctx->errbuf), "special row %lld (row %lld) not published%s", done,
                         (done + 1) * J.k, ctx->res_h[1].x == 2 ? " (kernel wait timeout)" : "");
                return SW_ECUDA;
            } else if (fe != cudaSuccess && fe != cudaErrorNotReady) {
                return bail(cuda_fail(ctx, fe, "fill kernel"));
            }
            if (dbg_host) {
                static double last = 0;
                if (hnow() - last > 1000.0) {
                    last = hnow();
                    fprintf(stderr, "[swb host] %.0f ms: done %lld/%lld released %llu sealed %d ready %d band %d colp %u copies %lld "
                            "evq %d sideq %d stq %d fill %d err %d\n", last, done,
                            nsp, *(volatile unsigned long long *)ctx->released.p, (int)sealed[slot], (int)row_ready(done),
                            band_of((done + 1) * J.k), ((volatile unsigned int *)ctx->colp[unit_lo(done)].p)[band_of((done + 1) * J.k)],
                            n_copies, (int)cudaEventQuery((*dview(ctx, sealdev[slot]).ev_row)[slot]), (int)cudaStreamQuery(ctx->side),
                            (int)cudaStreamQuery(st), (int)fe, (int)cudaPeekAtLastError());
                }
            }
            std::this_thread::yield();
        }
    }
    if ((rc = enqueue_results())) return bail(rc);
    if (dbg_host)
        fprintf(stderr, "[swb host] rows %lld copies %lld ring %lld fill_seen %.2f ms loop_end %.2f ms max_sink %.3f ms nstage %d\n",
                nsp, n_copies, R, h_fill, hnow(), h_sink_max, nstage);
    if (sink_rc) {
        bail(0);  // the kernels finish writing into released slots; no copy may land in a reused staging slot later
        return sink_rc;
    }
    for (int d = P - 1; d >= 0; d--) {
        CK(setdev(d));
        CK(cudaStreamSynchronize(d == 0 ? st : dview(ctx, d).stream));
    }
    CK(setdev(0));
    if (dbg_host)
        fprintf(stderr, "[swb host] synced %.2f ms; pre-launch: choose %.2f alloc %.2f encode %.2f\n", hnow(), h_choose,
                h_alloc, h_encode);
    if (ctx->res_h[1].x == 1) return SW_EALPHABET;
    if (ctx->res_h[1].x == 2) {
        snprintf(ctx->errbuf, sizeof(ctx->errbuf), "fill kernel: wait timeout (a neighbour stripe, entry or the special-row ring did not progress)");
        return SW_ECUDA;
    }
    // combine the entries' bests under the total order (reading S4)
    int4 r = ctx->res_h[0];
    long long reps = (long long)*(unsigned long long *)(ctx->res_h + 2);
    for (int d = 1; d < P; d++) {
        const int4 v = dview(ctx, d).res_h[0];
        reps += (long long)*(unsigned long long *)(dview(ctx, d).res_h + 2);
        if (J.local && v.x > 0 && (v.x > r.x || (v.x == r.x && (v.y < r.y || (v.y == r.y && v.z < r.z))))) r = v;
    }
    *res = r;

    float t01 = 0, t12 = 0, t23 = 0;
    cudaEventElapsedTime(&t01, ctx->ev[0], ctx->ev[1]);
    cudaEventElapsedTime(&t12, ctx->ev[1], ctx->ev[2]);
    cudaEventElapsedTime(&t23, ctx->ev[2], ctx->ev[3]);
    ctx->stats.encode_ms += t01;
    ctx->stats.fill_ms += t12;
    ctx->stats.reduce_ms += t23;
    ctx->stats.kernel_launches += 1 + (long long)P * (nseg + 1);
    ctx->stats.replays += reps;
    ctx->stats.special_rows += nsp;
    ctx->stats.special_bytes_d2h += bytes;
    ctx->stats.alpha = seg[0].use16 ? -V.alpha : V.alpha;  // negative: packed 16x2 kernel
    ctx->stats.patched = seg[0].patched ? 1 : 0;
    ctx->stats.warps = V.nw;
    ctx->stats.width = W;
    ctx->stats.grid = seg[0].grid[0];
    ctx->stats.devices = P;
    ctx->stats.sp_slots = (int32_t)R;
    ctx->stats.tail_alpha = nseg > 1 ? -seg[1].V->alpha : 0;
    ctx->stats.tail_warps = nseg > 1 ? seg[1].V->nw : 0;
    ctx->stats.tail_grid = nseg > 1 ? seg[1].grid[0] : 0;
    ctx->stats.tail_rows = nseg > 1 ? m - seg[1].row_base : 0;
    if (J.local) {
        // Stage 2 matches against these rows: resident in the ring, or in the host store
        S1Rows &S1 = ctx->s1;
        S1.resident = R >= nsp && !multi;
        S1.stored = store && !S1.resident;
        S1.valid = NS == 1 && !J.rank_mode && !rcyc && (S1.resident || S1.stored || nsp == 0);
        S1.m = J.m; S1.n = J.n; S1.k = J.k;
        S1.ma = J.ma; S1.mi = J.mi; S1.go = J.go; S1.ge = J.ge;
        S1.ld = ld[0]; S1.stride = stride[0];
    }
    return SW_OK;
}

static int stage1_common(sw_ctx *ctx, const unsigned char *dA, int64_t m, const unsigned char *dB, int64_t n,
                         int32_t ma, int32_t mi, int32_t go, int32_t ge, int64_t k, sw_row_sink sink, void *user,
                         cudaStream_t us, sw_result *out)
{
    Job J{};
    J.dA = dA; J.m = m; J.dB = dB; J.n = n;
    J.revA = J.revB = false;
    J.ma = ma; J.mi = mi; J.go = go; J.ge = ge;
    J.k = k; J.sink = sink; J.user = user;
    J.local = true;
    J.goal = 0;
    J.nv = (int)std::max<int64_t>(1, std::min<int64_t>(ctx->vstripes, n));
    J.epoch = ++ctx->epoch;
    int4 r;
    const int rc = run_job(ctx, J, us, &r);
    if (rc) return rc;
    out->score = r.x;
    out->i = r.y;
    out->j = r.z;
    return SW_OK;
}

static bool valid_common(sw_ctx *ctx, int64_t m, int64_t n, int64_t k, sw_row_sink sink, sw_result *out)
{
    if (!ctx || !out || m < 0 || n < 0 || k < 0) return false;
    if (m >= (1ll << 31) - (1 << 16) || n >= (1ll << 31) - (1 << 16)) return false;
    if (k > 0 && !sink) return false;
    return true;
}

static int upload(sw_ctx *ctx, const char *A, int64_t m, const char *B, int64_t n)
{
    int rc = grow(ctx, ctx->seq, (size_t)(m + n + 16));
    if (rc) return rc;
    if (m) CK(cudaMemcpyAsync(ctx->seq.p, A, (size_t)m, cudaMemcpyHostToDevice, ctx->stream));
    if (n) CK(cudaMemcpyAsync((char *)ctx->seq.p + m, B, (size_t)n, cudaMemcpyHostToDevice, ctx->stream));
    return SW_OK;
}

static void begin_stats(sw_ctx *ctx) { ctx->stats = sw_stats{}; }

extern "C" int sw_align_stage1(sw_ctx *ctx, const char *seqA, int64_t m, const char *seqB, int64_t n, int32_t match,
                               int32_t mismatch, int32_t gap_open, int32_t gap_ext, int64_t special_row_interval,
                               sw_row_sink sink, void *user, sw_result *out)
{
    if (!valid_common(ctx, m, n, special_row_interval, sink, out)) return SW_EINVAL;
    if ((m && !seqA) || (n && !seqB)) return SW_EINVAL;
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, m, n);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    const auto t0 = std::chrono::steady_clock::now();
    begin_stats(ctx);
    if (m == 0 || n == 0) {
        out->score = 0; out->i = 0; out->j = 0;
        return SW_OK;
    }
    CK(cudaEventRecord(ctx->ev[4], ctx->stream));
    if ((rc = upload(ctx, seqA, m, seqB, n))) return rc;
    rc = stage1_common(ctx, (const unsigned char *)ctx->seq.p, m, (const unsigned char *)ctx->seq.p + m, n, match,
                       mismatch, gap_open, gap_ext, special_row_interval, sink, user, nullptr, out);
    if (rc) return rc;
    float up = 0;
    cudaEventElapsedTime(&up, ctx->ev[4], ctx->ev[0]);
    ctx->stats.upload_ms = up;
    ctx->stats.total_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return SW_OK;
}

extern "C" int sw_align_stage1_dev(sw_ctx *ctx, const char *dseqA, int64_t m, const char *dseqB, int64_t n,
                                   int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext,
                                   int64_t special_row_interval, sw_row_sink sink, void *user, void *stream,
                                   sw_result *out)
{
    if (!valid_common(ctx, m, n, special_row_interval, sink, out)) return SW_EINVAL;
    if ((m && !dseqA) || (n && !dseqB)) return SW_EINVAL;
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, m, n);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    const auto t0 = std::chrono::steady_clock::now();
    begin_stats(ctx);
    if (m == 0 || n == 0) {
        out->score = 0; out->i = 0; out->j = 0;
        return SW_OK;
    }
    rc = stage1_common(ctx, (const unsigned char *)dseqA, m, (const unsigned char *)dseqB, n, match, mismatch,
                       gap_open, gap_ext, special_row_interval, sink, user, (cudaStream_t)stream, out);
    if (rc) return rc;
    ctx->stats.total_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return SW_OK;
}

// ---------------------------------------------------------------- multi-GPU column stripes

// Receive-area geometry valid for every kernel variant: rows cover the padded
// last band of the tallest band height, flags (band, warp) the finest split.
static size_t recv_rows(int64_t max_rows)
{
    int64_t rows = 0;  // the largest padded row count over the band heights (not all powers of two)
    for (int i = 0; i < NVARIANTS; i++) {
        const int64_t bh = (int64_t)variant_for(i).alpha * 32 * variant_for(i).nw;
        rows = std::max<int64_t>(rows, ((max_rows + bh - 1) / bh) * bh);
    }
    return (size_t)(rows + 2);
}
static size_t recv_flags(int64_t max_rows)
{
    size_t f = 0;
    for (int i = 0; i < NVARIANTS; i++) {
        const Variant &v = variant_for(i);
        const int64_t bh = (int64_t)v.alpha * 32 * v.nw;
        f = std::max<size_t>(f, (size_t)(((max_rows + bh - 1) / bh) * v.nw + 1));
    }
    return f;
}

extern "C" int sw_stripe_export(sw_ctx *ctx, int64_t max_rows, void *handle_out)
{
    if (!ctx || max_rows < 0 || !handle_out) return SW_EINVAL;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    // exact geometry: the left neighbour locates the flags from max_rows alone
    if (ctx->recv.base && (ctx->recv.rows != recv_rows(max_rows) || ctx->recv.flags != recv_flags(max_rows))) {
        cudaFree(ctx->recv.base);
        ctx->recv = RecvArea{};
    }
    int rc = grow_recv(ctx, ctx->recv, recv_rows(max_rows), recv_flags(max_rows));
    if (rc) return rc;
    cudaIpcMemHandle_t h;
    CK(cudaIpcGetMemHandle(&h, ctx->recv.base));
    memcpy(handle_out, &h, sizeof(h));
    return SW_OK;
}

extern "C" int sw_stripe_connect(sw_ctx *ctx, const void *right_handle, int64_t max_rows)
{
    if (!ctx) return SW_EINVAL;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    if (ctx->right_base) {
        cudaIpcCloseMemHandle(ctx->right_base);
        ctx->right_base = nullptr;
    }
    if (!right_handle) return SW_OK;
    cudaIpcMemHandle_t h;
    memcpy(&h, right_handle, sizeof(h));
    CK(cudaIpcOpenMemHandle(&ctx->right_base, h, cudaIpcMemLazyEnablePeerAccess));
    ctx->right_rows = recv_rows(max_rows);
    return SW_OK;
}

// ---------------------------------------------------------------- band-cyclic ranks (one process per GPU)

static size_t cyc_cols(int64_t max_cols) { return (size_t)(((max_cols + 63) / 64) * 64 + 5 * 64); }
static size_t cyc_bands(int64_t max_rows) { return (size_t)((max_rows + 2047) / 2048 + 4); }  // shortest band: 2048 rows

extern "C" int sw_cyclic_export(sw_ctx *ctx, int64_t max_rows, int64_t max_cols, void *handle_out)
{
    if (!ctx || max_rows < 0 || max_cols < 0 || !handle_out) return SW_EINVAL;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    const size_t cols = cyc_cols(max_cols), bands = cyc_bands(max_rows);
    if (!ctx->cin || ctx->cin_cols != cols || ctx->cin_bands != bands) {
        if (ctx->cin) cudaFree(ctx->cin);
        ctx->cin = nullptr;
        const size_t bytes = cols * sizeof(int2) + bands * sizeof(unsigned long long);
        if (cudaMalloc(&ctx->cin, bytes) != cudaSuccess) {
            cudaGetLastError();
            snprintf(ctx->errbuf, sizeof(ctx->errbuf), "cudaMalloc(%zu) for the band-cyclic area failed", bytes);
            return SW_ENOMEM;
        }
        CK(cudaMemset(ctx->cin, 0, bytes));  // progress tags start below every epoch
        ctx->cin_cols = cols;
        ctx->cin_bands = bands;
    }
    cudaIpcMemHandle_t h;
    CK(cudaIpcGetMemHandle(&h, ctx->cin));
    memcpy(handle_out, &h, sizeof(h));
    return SW_OK;
}

extern "C" int sw_cyclic_connect(sw_ctx *ctx, const void *next_handle, int64_t max_rows, int64_t max_cols)
{
    if (!ctx || !next_handle || max_rows < 0 || max_cols < 0) return SW_EINVAL;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    if (ctx->cout) {
        cudaIpcCloseMemHandle(ctx->cout);
        ctx->cout = nullptr;
    }
    cudaIpcMemHandle_t h;
    memcpy(&h, next_handle, sizeof(h));
    CK(cudaIpcOpenMemHandle(&ctx->cout, h, cudaIpcMemLazyEnablePeerAccess));
    ctx->cout_cols = cyc_cols(max_cols);
    ctx->cout_bands = cyc_bands(max_rows);
    return SW_OK;
}

extern "C" int32_t sw_cyclic_epoch(const sw_ctx *ctx) { return ctx ? ctx->pepoch : 0; }

extern "C" int sw_align_stage1_cyclic(sw_ctx *ctx, const char *dseqA, int64_t m, const char *dseqB, int64_t n,
                                      int32_t rank, int32_t world, int32_t epoch, int32_t match, int32_t mismatch,
                                      int32_t gap_open, int32_t gap_ext, int64_t special_row_interval,
                                      sw_row_sink sink, void *user, void *stream, sw_result *out)
{
    if (!valid_common(ctx, m, n, special_row_interval, sink, out)) return SW_EINVAL;
    if (!dseqA || !dseqB || m <= 0 || n <= 0 || world < 2 || world > 64 || rank < 0 || rank >= world) return SW_EINVAL;
    if (epoch <= ctx->pepoch) {
        snprintf(ctx->errbuf, sizeof(ctx->errbuf), "cyclic epoch %d not above this context's %d (sw_cyclic_epoch)", epoch, ctx->pepoch);
        return SW_EINVAL;
    }
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, m, n);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    const auto t0 = std::chrono::steady_clock::now();
    begin_stats(ctx);
    Job J{};
    J.dA = (const unsigned char *)dseqA; J.m = m; J.dB = (const unsigned char *)dseqB; J.n = n;
    J.ma = match; J.mi = mismatch; J.go = gap_open; J.ge = gap_ext;
    J.k = special_row_interval; J.sink = sink; J.user = user;
    J.local = true;
    J.nv = 1;
    J.rank_cyc = true;
    J.cyc_world = world;
    J.cyc_rank = rank;
    J.epoch = epoch;
    int4 r;
    rc = run_job(ctx, J, (cudaStream_t)stream, &r);
    if (rc) return rc;
    out->score = r.x;
    out->i = r.y;
    out->j = r.z;
    ctx->stats.total_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return SW_OK;
}

extern "C" int sw_plan(sw_ctx *ctx, int64_t m, int64_t n, int32_t match, int32_t mismatch, int32_t gap_open,
                       int32_t gap_ext, int64_t special_row_interval, int32_t world, int32_t *alpha, int32_t *warps)
{
    if (!ctx || !alpha || !warps || m < 0 || n < 0 || special_row_interval < 0 || world < 0) return SW_EINVAL;
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, m, n);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    Job J{};
    J.m = m; J.n = n;
    J.ma = match; J.mi = mismatch; J.go = gap_open; J.ge = gap_ext;
    J.k = special_row_interval;
    J.local = true;
    J.wide = std::abs((long long)match + gap_open + gap_ext) > 127 || std::abs((long long)mismatch + gap_open + gap_ext) > 127;
    J.rank_mode = world == 0;  // 0: a column-stripe rank; >= 1: a band-cyclic rank of `world`
    J.rank_cyc = world >= 1;
    J.cyc_world = std::max(1, (int)world);
    bool use16 = false;
    const Variant &V = choose_variant(ctx, J, &use16, J.rank_cyc ? J.cyc_world : 1);
    *alpha = use16 ? -V.alpha : V.alpha;
    *warps = V.nw;
    return SW_OK;
}

extern "C" int sw_align_stage1_stripe(sw_ctx *ctx, const char *dseqA, int64_t m, const char *dseqB, int64_t n,
                                      int64_t c_lo, int64_t c_hi, int32_t epoch, int32_t match, int32_t mismatch,
                                      int32_t gap_open, int32_t gap_ext, int64_t special_row_interval,
                                      sw_row_sink sink, void *user, void *stream, sw_result *out)
{
    if (!valid_common(ctx, m, n, special_row_interval, sink, out)) return SW_EINVAL;
    if (!dseqA || !dseqB || m <= 0 || c_lo < 0 || c_hi > n || c_hi <= c_lo || epoch <= 0) return SW_EINVAL;
    if (epoch <= ctx->stripe_epoch) {
        // the receive area's flags may hold any epoch up to stripe_epoch (equality test):
        // a repeated epoch would read stale borders (sw_stripe_epoch)
        snprintf(ctx->errbuf, sizeof(ctx->errbuf), "stripe epoch %d not above this context's %d", epoch, ctx->stripe_epoch);
        return SW_EINVAL;
    }
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, m, n);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    const auto t0 = std::chrono::steady_clock::now();
    begin_stats(ctx);
    Job J{};
    J.dA = (const unsigned char *)dseqA; J.m = m; J.dB = (const unsigned char *)dseqB; J.n = n;
    J.ma = match; J.mi = mismatch; J.go = gap_open; J.ge = gap_ext;
    J.k = special_row_interval; J.sink = sink; J.user = user;
    J.local = true;
    J.rank_mode = true;
    J.c_lo = c_lo;
    J.c_hi = c_hi;
    J.epoch = epoch;
    ctx->stripe_epoch = epoch;
    int4 r;
    rc = run_job(ctx, J, (cudaStream_t)stream, &r);
    if (rc) return rc;
    out->score = r.x;
    out->i = r.y;
    out->j = r.z;
    ctx->stats.total_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return SW_OK;
}

// ---------------------------------------------------------------- reverse pass

// Exact pruning: a cell (i', j') of the reverse matrix scores
// at most pmax*min(i',j') - [i' != j'](G_open + |i'-j'| G_ext), so a hit in rows
// <= L lies in columns <= J(L) = L + (pmax*L - G_open - goal)/G_ext.  The
// rectangle [1..L] x [1..J(L)] is closed under the recurrence's dependencies,
// so filling it exactly finds the first hit among rows <= L; L grows
// geometrically until a hit appears or L = i_end.
static int reverse_common(sw_ctx *ctx, const unsigned char *dA, int64_t i_end, const unsigned char *dB,
                          int64_t j_end, int32_t ma, int32_t mi, int32_t go, int32_t ge, int32_t goal,
                          cudaStream_t us, sw_result *out)
{
    const long long pmax = std::max(ma, mi);
    // First rectangle: twice the fewest rows a score of `goal` needs.  The fill
    // sweeps Jc columns band by band, so a short alignment (C2: 93 rows) costs
    // a few hundred columns instead of a whole band height of them.
    long long L = std::max<long long>(256, pmax > 0 ? 2 * ((goal + pmax - 1) / pmax) : i_end);
    for (;;) {
        // A rectangle of at least half the rows costs a large fraction of the
        // full one: take all rows at once instead of filling it twice (a
        // whole-length alignment starts with L = goal / pmax ~ i_end).
        L = std::min<long long>(L, i_end);
        if (2 * L >= i_end) L = i_end;
        long long Jc = j_end;
        if (ge > 0 && pmax > 0) {
            const long long slack = pmax * L - go - goal;
            const long long jl = slack < 0 ? L : L + slack / ge;
            Jc = std::min<long long>(j_end, std::max<long long>(jl, L));
        }
        Jc = std::min<long long>(Jc, j_end);
        Job J{};
        // reversed prefixes: row i' <-> S0[i_end - i'], column j' <-> S1[j_end - j'];
        // restricting to the first L rows / Jc columns of the reversed strings means
        // taking the LAST L (Jc) characters of the prefixes.
        J.dA = dA + (i_end - L);
        J.m = L;
        J.dB = dB + (j_end - Jc);
        J.n = Jc;
        J.revA = J.revB = true;
        J.ma = ma; J.mi = mi; J.go = go; J.ge = ge;
        J.k = 0; J.sink = nullptr; J.user = nullptr;
        J.local = false;
        J.goal = goal;
        J.nv = 1;
        J.epoch = ++ctx->epoch;
        int4 r;
        const int rc = run_job(ctx, J, us, &r);
        if (rc) return rc;
        if (r.w) {
            out->score = goal;
            out->i = i_end - r.y;
            out->j = j_end - r.z;
            return SW_OK;
        }
        if (L >= i_end) return SW_ENOTFOUND;  // the rectangle held every possible hit
        L = std::min<long long>(i_end, L * 4);
    }
}

extern "C" int sw_reverse_goal(sw_ctx *ctx, const char *seqA, int64_t i_end, const char *seqB, int64_t j_end,
                               int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext, int32_t goal,
                               sw_result *start_out)
{
    if (!ctx || !start_out || i_end < 0 || j_end < 0 || goal < 0) return SW_EINVAL;
    if ((i_end && !seqA) || (j_end && !seqB)) return SW_EINVAL;
    if (i_end >= (1ll << 31) - (1 << 16) || j_end >= (1ll << 31) - (1 << 16)) return SW_EINVAL;
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, i_end, j_end);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    const auto t0 = std::chrono::steady_clock::now();
    begin_stats(ctx);
    if (goal == 0) {
        start_out->score = 0; start_out->i = i_end; start_out->j = j_end;
        return SW_OK;
    }
    if (i_end == 0 || j_end == 0) return SW_ENOTFOUND;
    CK(cudaEventRecord(ctx->ev[4], ctx->stream));
    if ((rc = upload(ctx, seqA, i_end, seqB, j_end))) return rc;
    rc = reverse_common(ctx, (const unsigned char *)ctx->seq.p, i_end, (const unsigned char *)ctx->seq.p + i_end,
                        j_end, match, mismatch, gap_open, gap_ext, goal, nullptr, start_out);
    if (rc) return rc;
    ctx->stats.total_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return SW_OK;
}

extern "C" int sw_reverse_goal_dev(sw_ctx *ctx, const char *dseqA, int64_t i_end, const char *dseqB, int64_t j_end,
                                   int32_t match, int32_t mismatch, int32_t gap_open, int32_t gap_ext, int32_t goal,
                                   void *stream, sw_result *start_out)
{
    if (!ctx || !start_out || i_end < 0 || j_end < 0 || goal < 0) return SW_EINVAL;
    if ((i_end && !dseqA) || (j_end && !dseqB)) return SW_EINVAL;
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, i_end, j_end);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    begin_stats(ctx);
    if (goal == 0) {
        start_out->score = 0; start_out->i = i_end; start_out->j = j_end;
        return SW_OK;
    }
    if (i_end == 0 || j_end == 0) return SW_ENOTFOUND;
    return reverse_common(ctx, (const unsigned char *)dseqA, i_end, (const unsigned char *)dseqB, j_end, match,
                          mismatch, gap_open, gap_ext, goal, (cudaStream_t)stream, start_out);
}

// ---------------------------------------------------------------- Stage 2 (N1)

// Stage 2, partial traceback (readings S18-S22):
// from the end point back to the start point, one partition per special row.
// Each partition is a reverse GLOBAL fill of the TRANSPOSED problem -- DP
// rows j' = reversed S1 prefix (original columns j_c - j'), DP columns
// i' = reversed S0[r+1..i_c] -- so a band is a vertical strip of the original
// matrix (orthogonal execution) and the special row r is the last DP
// column, where the capture tiles run the goal-based matching; the band that
// holds the first event stops the bands after it.
static int stage2_common(sw_ctx *ctx, const unsigned char *dA, int64_t m, const unsigned char *dB, int64_t n,
                         int32_t ma, int32_t mi, int32_t go, int32_t ge, int64_t k, const sw_result *end,
                         cudaStream_t us, sw_crosspoint *out, int64_t cap, int64_t *count)
{
    const S1Rows &R = ctx->s1;
    if (!R.valid || R.m != m || R.n != n || R.k != k || R.ma != ma || R.mi != mi || R.go != go || R.ge != ge) {
        snprintf(ctx->errbuf, sizeof(ctx->errbuf),
                 "stage 2 needs the special rows of the last single-GPU sw_align_stage1 call with the same m, n, k and scoring");
        return SW_EINVAL;
    }
    cudaStream_t st = us ? us : ctx->stream;
    const int32_t *sp = (const int32_t *)ctx->sp[0].p;
    // H, F of special row r at column j (row 0 and column 0: H = 0, F = -inf):
    // from the device ring when every row stayed resident, else from the host
    // store (the SRA)
    auto fetch = [&](int64_t r, int64_t j, long long *h, long long *f) -> int {
        *h = 0;
        *f = NEG;
        if (r == 0 || j == 0) return SW_OK;
        if (!R.resident) {
            const std::vector<int32_t> &hr = ctx->host_rows[(size_t)(r / k - 1)];
            *h = hr[(size_t)(j - 1)];
            *f = hr[(size_t)(n + j - 1)];
            return SW_OK;
        }
        const int32_t *row = sp + (r / k - 1) * R.stride;
        CK(cudaMemcpyAsync(ctx->res_h + 3, row + j - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync((int32_t *)(ctx->res_h + 3) + 1, row + R.ld + j - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        *h = ((const int32_t *)(ctx->res_h + 3))[0];
        *f = ((const int32_t *)(ctx->res_h + 3))[1];
        return SW_OK;
    };
    std::vector<sw_crosspoint> L;
    sw_crosspoint C{end->i, end->j, end->score, 0};
    L.push_back(C);
    int rc;
    while (!(C.score == 0 && C.type == 0)) {
        if (C.i <= 0) return SW_ENOTFOUND;
        const int64_t r = k > 0 ? ((C.i - 1) / k) * k : 0, Lr = C.i - r;
        sw_crosspoint X{};
        bool found = false;
        {
            // strip j' = 0 is the reverse DP's boundary column: H' = F' = -(G_open + Lr G_ext) at row r
            long long hs, fs;
            if ((rc = fetch(r, C.j, &hs, &fs))) return rc;
            const long long rb = -((long long)go + Lr * (long long)ge);
            if (hs + rb == C.score) { X = sw_crosspoint{r, C.j, (int32_t)hs, 0}; found = true; }
            else if (fs > NEG / 2 && fs + rb + go == C.score) { X = sw_crosspoint{r, C.j, (int32_t)fs, 2}; found = true; }
        }
        if (!found) {
            if (C.j == 0) return SW_ENOTFOUND;
            Job J{};
            J.dA = dB; J.m = C.j; J.revA = true;      // DP rows: S1[C.j - j'] (0-based)
            J.dB = dA + r; J.n = Lr; J.revB = true;   // DP columns: S0[C.i - i'] (0-based)
            J.ma = ma; J.mi = mi; J.go = go; J.ge = ge;
            J.k = 0; J.sink = nullptr; J.user = nullptr;
            J.local = false;
            J.goal = C.score;
            J.nv = 1;
            J.epoch = ++ctx->epoch;
            J.hit_w = (int)(Lr - 1);  // start check strictly below row r
            J.anchor_gap = C.type == 2;
            J.match = true;
            J.mjc = C.j;
            if (r > 0 && R.resident) {
                J.mH = sp + (r / k - 1) * R.stride;
                J.mF = J.mH + R.ld;
            } else if (r > 0) {
                // special row r from the host store into HBM for the matching
                if ((rc = grow(ctx, ctx->s2row, (size_t)2 * n * sizeof(int32_t)))) return rc;
                CK(cudaMemcpyAsync(ctx->s2row.p, ctx->host_rows[(size_t)(r / k - 1)].data(), (size_t)2 * n * sizeof(int32_t),
                                   cudaMemcpyHostToDevice, st));
                J.mH = (const int *)ctx->s2row.p;
                J.mF = J.mH + n;
            }
            int4 res;
            const auto tj = std::chrono::steady_clock::now();
            const double f0 = ctx->stats.fill_ms;
            if ((rc = run_job(ctx, J, us, &res))) return rc;
            if (getenv("SWB_DEBUG_HOST"))
                fprintf(stderr, "[swb stage2] partition rows %lld..%lld jc %lld: run_job %.2f ms (fill %.2f ms) event (%d, %d)\n",
                        (long long)r, (long long)C.i, (long long)C.j,
                        std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tj).count(),
                        ctx->stats.fill_ms - f0, res.y, res.z);
            if (!res.w) return SW_ENOTFOUND;
            const int64_t jp = res.y, col = res.z;
            if (col <= Lr - 1) {
                X = sw_crosspoint{C.i - col, C.j - jp, 0, 0};  // the start point
            } else {
                long long hs, fs;
                if ((rc = fetch(r, C.j - jp, &hs, &fs))) return rc;
                X = col == Lr ? sw_crosspoint{r, C.j - jp, (int32_t)hs, 0} : sw_crosspoint{r, C.j - jp, (int32_t)fs, 2};
            }
        }
        L.push_back(X);
        C = X;
    }
    *count = (int64_t)L.size();
    for (int64_t q = 0; q < (int64_t)L.size() && q < cap; q++) out[q] = L[L.size() - 1 - q];
    return cap < (int64_t)L.size() ? SW_ERANGE : SW_OK;
}

static bool valid_stage2(const sw_ctx *ctx, int64_t m, int64_t n, int64_t k, const sw_result *end,
                         const sw_crosspoint *out, int64_t cap, const int64_t *count)
{
    if (!ctx || !end || !count || m < 0 || n < 0 || k < 0 || cap < 0 || (cap > 0 && !out)) return false;
    if (end->score < 0 || end->i < 0 || end->j < 0 || end->i > m || end->j > n) return false;
    return true;
}

extern "C" int sw_stage2(sw_ctx *ctx, const char *seqA, int64_t m, const char *seqB, int64_t n, int32_t match,
                         int32_t mismatch, int32_t gap_open, int32_t gap_ext, int64_t special_row_interval,
                         const sw_result *end, sw_crosspoint *out, int64_t cap, int64_t *count)
{
    if (!valid_stage2(ctx, m, n, special_row_interval, end, out, cap, count)) return SW_EINVAL;
    if ((m && !seqA) || (n && !seqB)) return SW_EINVAL;
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, m, n);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    const auto t0 = std::chrono::steady_clock::now();
    begin_stats(ctx);
    if ((rc = upload(ctx, seqA, m, seqB, n))) return rc;
    rc = stage2_common(ctx, (const unsigned char *)ctx->seq.p, m, (const unsigned char *)ctx->seq.p + m, n, match,
                       mismatch, gap_open, gap_ext, special_row_interval, end, nullptr, out, cap, count);
    ctx->stats.total_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return rc;
}

extern "C" int sw_stage2_dev(sw_ctx *ctx, const char *dseqA, int64_t m, const char *dseqB, int64_t n, int32_t match,
                             int32_t mismatch, int32_t gap_open, int32_t gap_ext, int64_t special_row_interval,
                             const sw_result *end, void *stream, sw_crosspoint *out, int64_t cap, int64_t *count)
{
    if (!valid_stage2(ctx, m, n, special_row_interval, end, out, cap, count)) return SW_EINVAL;
    if ((m && !dseqA) || (n && !dseqB)) return SW_EINVAL;
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, m, n);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    begin_stats(ctx);
    return stage2_common(ctx, (const unsigned char *)dseqA, m, (const unsigned char *)dseqB, n, match, mismatch,
                         gap_open, gap_ext, special_row_interval, end, (cudaStream_t)stream, out, cap, count);
}

// ---------------------------------------------------------------- Stages 3-5 (N2/N3)

#include "sw_mm.cuh"

// Stages 3-5: from the crosspoints L_2 of Stage 2,
// split every partition larger than MM_TB_CELLS by Myers-Miller with balanced
// splitting on the GPU (one warp per partition, one launch per level), then
// align every small partition with a full traceback (one warp each, one
// launch) and concatenate.  The GAP_1 / GAP_2 lists are the maximal
// runs of the concatenated moves.
static int align_common(sw_ctx *ctx, const unsigned char *dA, int64_t m, const unsigned char *dB, int64_t n,
                        int32_t ma, int32_t mi, int32_t go, int32_t ge, int64_t k, cudaStream_t us,
                        sw_alignment *out, sw_gap *gap1, int64_t cap1, sw_gap *gap2, int64_t cap2)
{
    cudaStream_t st = us ? us : ctx->stream;
    sw_result best{};
    auto tnow = std::chrono::steady_clock::now;
    auto ms = [](std::chrono::steady_clock::time_point a, std::chrono::steady_clock::time_point b) {
        return std::chrono::duration<double, std::milli>(b - a).count();
    };
    const auto t0 = tnow();
    // Stage 1; the special rows stay resident in HBM for Stage 2 (no host sink)
    int rc = stage1_common(ctx, dA, m, dB, n, ma, mi, go, ge, k, nullptr, nullptr, us, &best);
    if (rc) return rc;
    *out = sw_alignment{};
    out->score = best.score;
    out->ms_stage1 = ms(t0, tnow());
    if (best.score == 0) return SW_OK;
    // Stage 2: crosspoints on the special rows
    std::vector<sw_crosspoint> L(64);
    int64_t cnt = 0;
    for (;;) {
        rc = stage2_common(ctx, dA, m, dB, n, ma, mi, go, ge, k, &best, us, L.data(), (int64_t)L.size(), &cnt);
        if (rc == SW_ERANGE && cnt > (int64_t)L.size()) { L.resize((size_t)cnt); continue; }
        if (rc) return rc;
        break;
    }
    L.resize((size_t)cnt);
    const auto t2 = tnow();
    out->ms_stage2 = ms(t0, t2) - out->ms_stage1;
    std::vector<MMPart> parts;
    for (size_t q = 0; q + 1 < L.size(); q++) {
        MMPart p{};
        p.i_s = (int)L[q].i; p.j_s = (int)L[q].j; p.i_e = (int)L[q + 1].i; p.j_e = (int)L[q + 1].j;
        p.t_s = L[q].type; p.t_e = L[q + 1].type;
        p.score = L[q + 1].score - L[q].score;
        parts.push_back(p);
    }
    MMArgs g{};
    g.A = dA; g.B = dB;
    g.ma = ma; g.mi = mi; g.go = go; g.ge = ge; g.gf = go + ge;
    for (int x = 0; x < 4; x++) {
        uint32_t wv = 0;
        for (int y = 0; y < 4; y++) wv |= (uint32_t)(uint8_t)(int8_t)((x == y ? ma : mi) + g.gf) << (8 * y);
        g.prof[x] = wv;
    }
    g.pm_gf = ma + g.gf;
    g.pn_gf = mi + g.gf;
    g.wide = std::abs((long long)ma + g.gf) > 127 || std::abs((long long)mi + g.gf) > 127;
    auto cells = [](const MMPart &p) { return (long long)(p.i_e - p.i_s) * (long long)(p.j_e - p.j_s); };
    const int WPB = 8;  // warps per block
    if ((rc = grow(ctx, ctx->mm_err, sizeof(int)))) return rc;
    CK(cudaMemsetAsync(ctx->mm_err.p, 0, sizeof(int), st));
    g.err = (int *)ctx->mm_err.p;
    g.timeout_ns = ctx->timeout_ns;
    // Stage 3/4: balanced Myers-Miller splitting until every partition is small.
    // Partitions whose split line is at least MM_CTA_ROWS away from C_s go to the
    // CTA kernel (MM_NWP warps on the chunks), the rest one warp each.
    long long MM_CTA_ROWS = 4ll * MM_CHUNK;
    if (const char *e = getenv("SWB_MM_CTA_ROWS")) MM_CTA_ROWS = atoll(e);  // tuning
    int levels = 0;
    for (;; levels++) {
        std::vector<size_t> big;
        for (size_t q = 0; q < parts.size(); q++)
            if (cells(parts[q]) > MM_TB_CELLS) big.push_back(q);
        if (big.empty()) break;
        // CTA partitions first (blocks 0..ncta-1), then warp partitions
        std::vector<MMPart> bp;
        std::vector<size_t> order;
        long long scr = 0;
        int ncta = 0;
        for (int pass = 0; pass < 2; pass++)
            for (size_t q : big) {
                const MMPart &P = parts[q];
                const long long hh = P.i_e - P.i_s, ww = P.j_e - P.j_s;
                const long long H = std::max(hh, ww), Wd = std::min(hh, ww);
                const bool cta = H / 2 >= MM_CTA_ROWS;
                if (cta != (pass == 0)) continue;
                MMPart c = P;
                c.off = scr;
                scr += (cta ? (2 * (MM_NWP + 1) + 2) : 3) * (Wd + 1);  // CTA: two lines + a ring per pass
                bp.push_back(c);
                order.push_back(q);
                ncta += cta;
            }
        if ((rc = grow(ctx, ctx->mm_parts, bp.size() * sizeof(MMPart)))) return rc;
        if ((rc = grow(ctx, ctx->mm_scratch, (size_t)scr * sizeof(int2)))) return rc;
        if ((rc = grow(ctx, ctx->mm_res, bp.size() * sizeof(MMRes)))) return rc;
        CK(cudaMemcpyAsync(ctx->mm_parts.p, bp.data(), bp.size() * sizeof(MMPart), cudaMemcpyHostToDevice, st));
        g.scratch = (int2 *)ctx->mm_scratch.p;
        if (ncta > 0) {
            if ((rc = grow(ctx, ctx->mm_cnt, (size_t)ncta * sizeof(int)))) return rc;
            CK(cudaMemsetAsync(ctx->mm_cnt.p, 0, (size_t)ncta * sizeof(int), st));
            g.cnt = (int *)ctx->mm_cnt.p;
            g.nparts = ncta;
            g.parts = (const MMPart *)ctx->mm_parts.p;
            g.res = (MMRes *)ctx->mm_res.p;
            sw_mm_split_cta_kernel<<<2 * ncta, 32 * MM_NWP, 0, st>>>(g);  // forward and reverse pass CTAs
            CK(cudaGetLastError());
            ctx->stats.kernel_launches++;
        }
        if ((int)bp.size() > ncta) {
            g.nparts = (int)bp.size() - ncta;
            g.parts = (const MMPart *)ctx->mm_parts.p + ncta;
            g.res = (MMRes *)ctx->mm_res.p + ncta;
            sw_mm_split_kernel<<<(g.nparts + WPB - 1) / WPB, 32 * WPB, 0, st>>>(g);
            CK(cudaGetLastError());
            ctx->stats.kernel_launches++;
        }
        std::vector<MMRes> resv(bp.size());
        int merr = 0;
        CK(cudaMemcpyAsync(resv.data(), ctx->mm_res.p, resv.size() * sizeof(MMRes), cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(&merr, ctx->mm_err.p, sizeof(int), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        if (merr) {
            snprintf(ctx->errbuf, sizeof(ctx->errbuf), "Myers-Miller split: spin-wait timeout");
            return SW_ECUDA;
        }
        if (getenv("SWB_DEBUG_HOST"))
            fprintf(stderr, "[swb mm] level %d: %zu partitions split (%d on CTAs), t=%.1f ms\n", levels, bp.size(),
                    ncta, ms(t2, tnow()));
        std::vector<MMRes> res(parts.size());
        for (size_t q = 0; q < order.size(); q++) res[order[q]] = resv[q];
        std::vector<MMPart> next;
        size_t bi = 0;
        for (size_t q = 0; q < parts.size(); q++) {
            if (bi < big.size() && big[bi] == q) {
                bi++;
                const MMRes &r = res[q];
                if (r.type < 0) {
                    snprintf(ctx->errbuf, sizeof(ctx->errbuf), "Myers-Miller split found no junction (partition %zu)", q);
                    return SW_ENOTFOUND;
                }
                MMPart a = parts[q], b = parts[q];
                a.i_e = r.i; a.j_e = r.j; a.t_e = r.type; a.score = r.sub;
                b.i_s = r.i; b.j_s = r.j; b.t_s = r.type; b.score = parts[q].score - r.sub;
                next.push_back(a);
                next.push_back(b);
            } else {
                next.push_back(parts[q]);
            }
        }
        parts.swap(next);
        if (levels > 128) return SW_ECUDA;
    }
    const auto t3 = tnow();
    out->ms_mm = ms(t2, t3);
    // Stage 5: full traceback of every (small) partition
    long long oc = 0, om = 0, os = 0;
    for (MMPart &p : parts) {
        const long long h = p.i_e - p.i_s, w = p.j_e - p.j_s;
        p.off_c = oc;
        p.off_m = om;
        p.off = os;
        oc += (w + 1) * ((h + 7) / 8);
        om += h + w;
        os += w + 1;
    }
    if ((rc = grow(ctx, ctx->mm_parts, parts.size() * sizeof(MMPart)))) return rc;
    if ((rc = grow(ctx, ctx->mm_scratch, (size_t)std::max(1ll, os) * sizeof(int2)))) return rc;
    if ((rc = grow(ctx, ctx->mm_codes, (size_t)std::max(1ll, oc) * sizeof(unsigned int)))) return rc;
    if ((rc = grow(ctx, ctx->mm_moves, (size_t)std::max(1ll, om)))) return rc;
    if ((rc = grow(ctx, ctx->mm_res, parts.size() * sizeof(int)))) return rc;
    CK(cudaMemcpyAsync(ctx->mm_parts.p, parts.data(), parts.size() * sizeof(MMPart), cudaMemcpyHostToDevice, st));
    g.nparts = (int)parts.size();
    g.parts = (const MMPart *)ctx->mm_parts.p;
    g.scratch = (int2 *)ctx->mm_scratch.p;
    g.codes = (unsigned int *)ctx->mm_codes.p;
    g.moves = (char *)ctx->mm_moves.p;
    g.nmoves = (int *)ctx->mm_res.p;
    sw_mm_tb_kernel<<<(g.nparts + WPB - 1) / WPB, 32 * WPB, 0, st>>>(g);
    CK(cudaGetLastError());
    ctx->stats.kernel_launches++;
    std::vector<char> mv((size_t)std::max(1ll, om));
    std::vector<int> nm(parts.size());
    CK(cudaMemcpyAsync(mv.data(), ctx->mm_moves.p, (size_t)om, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(nm.data(), ctx->mm_res.p, nm.size() * sizeof(int), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    // concatenate and run-length encode into GAP_1 (gaps in S0) / GAP_2 (gaps in S1)
    out->i0 = L.front().i; out->j0 = L.front().j;
    out->i1 = best.i; out->j1 = best.j;
    out->partitions = (int64_t)parts.size();
    out->mm_levels = levels;
    int64_t i = out->i0, j = out->j0, n1 = 0, n2 = 0;
    char prev = 0;
    for (size_t q = 0; q < parts.size(); q++) {
        const MMPart &p = parts[q];
        const long long len = (long long)(p.i_e - p.i_s) + (p.j_e - p.j_s);
        const char *s = mv.data() + p.off_m + (len - nm[q]);
        for (int x = 0; x < nm[q]; x++) {
            const char c = s[x];
            if (c == 'I') {
                if (prev == 'I') { if (n1 <= cap1 && n1 > 0) gap1[n1 - 1].len++; }
                else { if (n1 < cap1) gap1[n1] = sw_gap{i, j, 1}; n1++; }
                j++;
            } else if (c == 'D') {
                if (prev == 'D') { if (n2 <= cap2 && n2 > 0) gap2[n2 - 1].len++; }
                else { if (n2 < cap2) gap2[n2] = sw_gap{i, j, 1}; n2++; }
                i++;
            } else {
                i++;
                j++;
            }
            prev = c;
        }
    }
    out->n_gap1 = n1;
    out->n_gap2 = n2;
    out->ms_stage5 = ms(t3, tnow());
    if (i != out->i1 || j != out->j1) {
        snprintf(ctx->errbuf, sizeof(ctx->errbuf), "alignment ends at (%lld, %lld), expected (%lld, %lld)",
                 (long long)i, (long long)j, (long long)out->i1, (long long)out->j1);
        return SW_ECUDA;
    }
    return (n1 > cap1 || n2 > cap2) ? SW_ERANGE : SW_OK;
}

extern "C" int sw_align(sw_ctx *ctx, const char *seqA, int64_t m, const char *seqB, int64_t n, int32_t match,
                        int32_t mismatch, int32_t gap_open, int32_t gap_ext, int64_t special_row_interval,
                        sw_alignment *out, sw_gap *gap1, int64_t cap1, sw_gap *gap2, int64_t cap2)
{
    if (!ctx || !out || m < 0 || n < 0 || special_row_interval < 0 || cap1 < 0 || cap2 < 0) return SW_EINVAL;
    if ((cap1 > 0 && !gap1) || (cap2 > 0 && !gap2)) return SW_EINVAL;
    if (m >= (1ll << 31) - (1 << 16) || n >= (1ll << 31) - (1 << 16)) return SW_EINVAL;
    if ((m && !seqA) || (n && !seqB)) return SW_EINVAL;
    int rc = check_scoring(match, mismatch, gap_open, gap_ext, m, n);
    if (rc) return rc;
    if (cudaSetDevice(ctx->device) != cudaSuccess) return SW_ECUDA;
    const auto t0 = std::chrono::steady_clock::now();
    begin_stats(ctx);
    *out = sw_alignment{};
    if (m == 0 || n == 0) return SW_OK;
    if ((rc = upload(ctx, seqA, m, seqB, n))) return rc;
    rc = align_common(ctx, (const unsigned char *)ctx->seq.p, m, (const unsigned char *)ctx->seq.p + m, n, match,
                      mismatch, gap_open, gap_ext, special_row_interval, nullptr, out, gap1, cap1, gap2, cap2);
    ctx->stats.total_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return rc;
}
