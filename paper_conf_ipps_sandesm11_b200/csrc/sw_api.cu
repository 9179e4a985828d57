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
};

template <int NW, int W, bool COOP, int NS>
static void packed_name(Variant &v)
{
    snprintf(v.packed_name, sizeof(v.packed_name), "_ZN3swb16sw_fill16_kernelILi%dELi%dELb%dELi%dELb0ELb1EEEvNS_8FillArgsE",
             NW, W, COOP ? 1 : 0, NS);
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
    if constexpr (ALPHA == 32 || ALPHA == 30) {
        // packed kernel only (16 or 15 slots per lane); int32 work falls back to the default geometry
        constexpr int NS = ALPHA / 2;
        v.packed_fn = (const void *)&sw_fill16_kernel<NW, W, COOP, NS, SPLIT>;
        v.io_warps = COOP ? 0 : 1;
        v.smem16 = Fill16<NW, W, NS, SPLIT>::smem_bytes();
        if constexpr (!SPLIT) packed_name<NW, W, COOP, NS>(v);
        if constexpr (ALPHA == 32 && NW == 8 && !COOP && !SPLIT) {
            // the reverse pass (a8) on the packed kernel
            v.packed_global_fn = (const void *)&sw_fill16_kernel<NW, W, false, 16, false, false>;
            snprintf(v.packed_global_name, sizeof(v.packed_global_name),
                     "_ZN3swb16sw_fill16_kernelILi%dELi%dELb0ELi16ELb0ELb0EEEvNS_8FillArgsE", NW, W);
        }
        return v;
    } else {
        v.local_fn = (const void *)&sw_fill_kernel<ALPHA, NW, W, true>;
        v.global_fn = (const void *)&sw_fill_kernel<ALPHA, NW, W, false>;
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
            if constexpr (NW == 8) {
                // Stage-2 partitions (global mode with matching) on the packed kernel
                v.packed_global_fn = (const void *)&sw_fill16_kernel<NW, W, false, 8, false, false>;
                snprintf(v.packed_global_name, sizeof(v.packed_global_name),
                         "_ZN3swb16sw_fill16_kernelILi%dELi%dELb0ELi8ELb0ELb0EEEvNS_8FillArgsE", NW, W);
            }
        }
        v.smem16 = Fill16<NW, W>::smem_bytes();
    }
    return v;
}

static constexpr int DEFAULT_VARIANT = 1;  // (alpha 16, 8 warps, W 64): fastest on C2/C3
static constexpr int NVARIANTS = 14;
static constexpr int NINT32_VARIANTS = 8;  // variants 0..7 have int32 kernels; 8.. are packed-only (alpha 32)

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

// Where the special rows of the last Stage-1 call live (for Stage 2).
struct S1Rows {
    bool valid = false;
    int64_t m = 0, n = 0, k = 0;
    int32_t ma = 0, mi = 0, go = 0, ge = 0;
    int64_t ld = 0, stride = 0;  // row q at sp[0] + q * stride: H[0..n), F at + ld
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

#if defined(SWB_PATCH_CUBIN) && !defined(__CUDA_ARCH__)
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
    const void *fn[4][NVARIANTS] = {};  // [packed, int32 local, int32 global, packed global][variant]
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
    cudaStream_t stream = nullptr, side = nullptr;
    cudaEvent_t ev[6] = {};
    std::vector<cudaEvent_t> ev_row;  // one per staging slot: the slot's final copy is done
    int nstage = 2;
    DevBuf seq, a2, b2, misc, slots, dbg;
    DevBuf mm_parts, mm_scratch, mm_res, mm_codes, mm_moves, mm_err;  // Stages 3-5
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
    if (cudaHostAlloc(&b.p, std::max<size_t>(bytes, 64), mapped ? cudaHostAllocMapped : cudaHostAllocDefault) != cudaSuccess) {
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

extern "C" int sw_init(const int *device_ids, int n_devices, sw_ctx **out)
{
    if (!out || n_devices != 1 || !device_ids) return SW_EINVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev <= 0) { cudaGetLastError(); return SW_ECUDA; }
    if (device_ids[0] < 0 || device_ids[0] >= ndev) return SW_EINVAL;
    sw_ctx *ctx = new sw_ctx();
    ctx->device = device_ids[0];
    int rc = SW_OK;
    do {
        cudaError_t e;
        if ((e = cudaSetDevice(ctx->device)) != cudaSuccess) { rc = cuda_fail(ctx, e, "cudaSetDevice"); break; }
        cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, ctx->device);
        if ((e = cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking)) != cudaSuccess) { rc = cuda_fail(ctx, e, "stream"); break; }
        if ((e = cudaStreamCreateWithFlags(&ctx->side, cudaStreamNonBlocking)) != cudaSuccess) { rc = cuda_fail(ctx, e, "stream"); break; }
        for (auto &ev : ctx->ev)
            if ((e = cudaEventCreate(&ev)) != cudaSuccess) { rc = cuda_fail(ctx, e, "event"); break; }
        if (rc) break;
        if ((e = cudaHostAlloc(&ctx->res_h, 4 * sizeof(int4), cudaHostAllocDefault)) != cudaSuccess) { rc = SW_ENOMEM; break; }
        for (int i = 0; i < NVARIANTS; i++) {
            const Variant &v = variant_for(i);
            if (v.local_fn) cudaFuncSetAttribute(v.local_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem);
            if (v.global_fn) cudaFuncSetAttribute(v.global_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem);
            if (v.packed_fn) cudaFuncSetAttribute(v.packed_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem16);
            if (v.packed_global_fn)
                cudaFuncSetAttribute(v.packed_global_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem16);
        }
        if ((e = cudaGetLastError()) != cudaSuccess) { rc = cuda_fail(ctx, e, "cudaFuncSetAttribute"); break; }
        if (const char *ov = getenv("SWB_VARIANT")) ctx->variant_override = atoi(ov);
        if (const char *vs = getenv("SWB_VSTRIPES")) ctx->vstripes = std::max(1, std::min(MAX_STRIPES, atoi(vs)));
        if (const char *to = getenv("SWB_TIMEOUT_S")) ctx->timeout_ns = (long long)(atof(to) * 1e9);
        if (const char *pk = getenv("SWB_PACKED")) ctx->packed = atoi(pk);
        if (const char *pt = getenv("SWB_PATCH")) ctx->patch = atoi(pt);
    } while (0);
    if (rc) { sw_shutdown(ctx); return rc; }
    *out = ctx;
    return SW_OK;
}

extern "C" void sw_shutdown(sw_ctx *ctx)
{
    if (!ctx) return;
    cudaSetDevice(ctx->device);
    if (ctx->stream) cudaStreamSynchronize(ctx->stream);
    if (ctx->side) cudaStreamSynchronize(ctx->side);
    for (DevBuf *b : {&ctx->seq, &ctx->a2, &ctx->b2, &ctx->misc, &ctx->slots, &ctx->dbg, &ctx->capbuf, &ctx->mm_parts,
                      &ctx->mm_scratch, &ctx->mm_res, &ctx->mm_codes, &ctx->mm_moves, &ctx->mm_err})
        if (b->p) cudaFree(b->p);
    for (int s = 0; s < MAX_STRIPES; s++) {
        for (DevBuf *b : {&ctx->rowb[s], &ctx->progress[s], &ctx->sp[s]})
            if (b->p) cudaFree(b->p);
        if (ctx->flags[s].p) cudaFreeHost(ctx->flags[s].p);
        if (ctx->colp[s].p) cudaFreeHost(ctx->colp[s].p);
        if (ctx->vrecv[s].base) cudaFree(ctx->vrecv[s].base);
    }
    for (auto &P : ctx->patched)
        if (P.lib) cudaLibraryUnload(P.lib);
    if (ctx->right_base) cudaIpcCloseMemHandle(ctx->right_base);
    if (ctx->recv.base) cudaFree(ctx->recv.base);
    if (ctx->stage.p) cudaFreeHost(ctx->stage.p);
    if (ctx->res_h) cudaFreeHost(ctx->res_h);
    for (auto &ev : ctx->ev)
        if (ev) cudaEventDestroy(ev);
    for (auto &ev : ctx->ev_row)
        if (ev) cudaEventDestroy(ev);
    if (ctx->stream) cudaStreamDestroy(ctx->stream);
    if (ctx->side) cudaStreamDestroy(ctx->side);
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
    if (llabs(ma + gf) > 127 || llabs(mi + gf) > 127) return SW_EINVAL;  // int8 profile
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
    // kind 0: packed local, 3: packed global (the kernels in the patched image);
    // 1, 2: int32 local/global (not patched)
    if ((kind != 0 && kind != 3) || !ctx->patch) return nullptr;
    const char *name = kind == 0 ? V.packed_name : V.packed_global_name;
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
                                 (int)(kind == 0 || kind == 3 ? V.smem16 : V.smem)) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        P->fn[kind][vidx] = (const void *)k;
    }
    return P->fn[kind][vidx];
}

static const Variant &choose_variant(sw_ctx *ctx, const Job &J, bool *use16)
{
    const long long pmax_abs = std::max(std::abs(J.ma), std::abs(J.mi));
    // packed preconditions: local mode, special rows at strip
    // bottoms, and a warp's live values (32 alpha rows x ~130 columns of
    // Manhattan distance, each step <= p_max + G_first apart) inside the 16-bit frame
    auto packed_ok = [&](const Variant &V) {
        const long long span = 32ll * V.alpha + 140;
        return ctx->packed && J.local && V.packed_fn && (J.k == 0 || J.k % V.alpha == 0) &&
               span * (pmax_abs + J.go + J.ge) + 1024 < 30000;
    };
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
    // profiles/r01_variants.txt; earlier entries win near-ties (3 %)
    static const Candidate cands[] = {
        {DEFAULT_VARIANT, false, 4.24e6, 4.24e6},  // int32, 8 warps + I/O warp
        {1, true, 8.08e6, 7.74e6},                 // packed alpha 16, 8 warps + I/O warp
        {8, true, 4.25e6, 7.86e6},                 // packed alpha 32, 4 warps + I/O warp (2 CTAs/SM)
        {13, true, 4.45e6, 8.17e6},                // packed alpha 30, 4 warps + I/O warp (2 CTAs/SM)
        {10, true, 4.49e6, 4.49e6},                // packed alpha 32, 8 warps + I/O warp
        {5, true, 4.03e6, 4.03e6},                 // packed alpha 16, 15 warps + I/O warp
        {6, true, 3.87e6, 3.87e6},                 // packed alpha 16, 16 warps, cooperative I/O
    };
    double best_t = 1e300;
    int best = 0;
    for (int c = 0; c < (int)(sizeof(cands) / sizeof(cands[0])); c++) {
        const Candidate &C = cands[c];
        const Variant &V = variant_for(C.variant);
        if (C.packed && !packed_ok(V)) continue;
        if (!C.packed && !J.local) { best = c; break; }  // reverse pass: int32 only
        const void *fn = C.packed ? V.packed_fn : V.local_fn;
        if (!fn) continue;
        int per_sm = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, V.nw * 32 + (C.packed ? V.io_warps : 1) * 32,
                                                      C.packed ? V.smem16 : V.smem);
        const long long P = (long long)std::max(1, per_sm) * ctx->num_sms;
        const long long bh = (long long)V.alpha * 32 * V.nw;
        const long long nb = std::max<long long>(1, (J.m + bh - 1) / bh);
        const double cps = nb <= ctx->num_sms ? C.cps_solo : C.cps_full;
        double t = model_fill_time(nb, P, std::max<long long>(J.n, 1), (2ll * V.nw + 2) * V.w, cps);
        // special rows that are not band bottoms are written by the compute
        // warps (SP1 tiles) instead of the I/O warp: measured +7.7 % on C2
        // (variant 8 at k = 3840 vs 4096, profiles/r01_fill_a30.txt)
        if (J.k > 0 && J.k < J.m && J.k % bh != 0) t *= 1.077;
        if (t < best_t * 0.97) {
            best_t = t;
            best = c;
        }
    }
    *use16 = cands[best].packed;
    return variant_for(cands[best].variant);
}

static int run_job(sw_ctx *ctx, const Job &J, cudaStream_t user_stream, int4 *res)
{
    const auto h0 = std::chrono::steady_clock::now();
    if (J.local) ctx->s1.valid = false;
    double hck[6] = {0, 0, 0, 0, 0, 0};
    auto hnow = [&]() { return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - h0).count(); };
    bool use16 = false;
    const Variant &V = choose_variant(ctx, J, &use16);
    hck[0] = hnow();
    const int W = V.w;
    const int BH = V.alpha * 32 * V.nw;
    const int m = (int)J.m, n = (int)J.n;
    const int nb = (m + BH - 1) / BH;
    const long long wa = (J.m + 15) / 16 + 2, wb = (J.n + 15) / 16 + 2;
    const int NS = J.rank_mode ? 1 : J.nv;
    int rc;

    // stripe geometry
    long long col0[MAX_STRIPES], wid[MAX_STRIPES];
    if (J.rank_mode) {
        col0[0] = J.c_lo;
        wid[0] = J.c_hi - J.c_lo;
    } else {
        for (int s = 0; s < NS; s++) {
            col0[s] = (long long)n * s / NS;
            wid[s] = (long long)n * (s + 1) / NS - col0[s];
        }
    }
    for (int s = 0; s < NS; s++)
        if (wid[s] <= 0) {
            snprintf(ctx->errbuf, sizeof(ctx->errbuf), "stripe %d is empty (n=%d, stripes=%d)", s, n, NS);
            return SW_EINVAL;
        }

    if ((rc = grow(ctx, ctx->a2, wa * 4))) return rc;
    if ((rc = grow(ctx, ctx->b2, wb * 4))) return rc;
    if ((rc = grow(ctx, ctx->misc, 256))) return rc;
    if (J.match && (rc = grow(ctx, ctx->capbuf, ((size_t)nb * BH + 2) * sizeof(int2)))) return rc;
    const size_t border_rows = (size_t)nb * BH + 2;
    const size_t border_flags = (size_t)nb * V.nw + 1;
    for (int s = 0; s < NS; s++) {
        const int npad = (int)((wid[s] + W - 1) / W) * W;
        const int NT = npad / W + (use16 ? 1 : V.skew_tiles);
        if ((rc = grow(ctx, ctx->rowb[s], (size_t)(NT * W + 2 * W) * sizeof(int2)))) return rc;
        if ((rc = grow(ctx, ctx->progress[s], (size_t)(nb + 1) * sizeof(int)))) return rc;
        if (!J.rank_mode && s > 0)
            if ((rc = grow_recv(ctx, ctx->vrecv[s], border_rows, border_flags))) return rc;
    }
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
    const void *fill_fn = use16 ? (J.local ? V.packed_fn : V.packed_global_fn) : (J.local ? V.local_fn : V.global_fn);
    const size_t fill_smem = use16 ? V.smem16 : V.smem;
    bool patched = false;
    if (const void *pf = patched_kernel(ctx, V, J.ge, J.go + J.ge, use16 ? (J.local ? 0 : 3) : J.local ? 1 : 2)) {
        fill_fn = pf;
        patched = true;
    }
    const int block = V.nw * 32 + (use16 ? V.io_warps : 1) * 32;
    int blocks_per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, fill_fn, block, fill_smem);
    if (blocks_per_sm < 1) blocks_per_sm = 1;
    // every CTA of every stripe must be co-resident (stripes wait on each other)
    int per_stripe = std::max(1, std::min(nb, blocks_per_sm * ctx->num_sms / NS));
    if (const char *g = getenv("SWB_GRID")) per_stripe = std::max(1, std::min(per_stripe, atoi(g) / NS));
    if (ctx->grid_cap > 0) per_stripe = std::max(1, std::min(per_stripe, ctx->grid_cap / NS));
    const int grid = per_stripe * NS;
    hck[1] = hnow();
    if ((rc = grow(ctx, ctx->slots, (size_t)grid * sizeof(int4)))) return rc;

    // special rows: all of them stay resident on the device (180 GB HBM) and
    // are streamed to the host as bands complete.
    const long long nsp = (J.local && J.k > 0) ? J.m / J.k : 0;
    int ld[MAX_STRIPES];
    long long stride[MAX_STRIPES];
    size_t row_ints = 0;
    for (int s = 0; s < NS; s++) {
        ld[s] = (int)((wid[s] + 31) / 32) * 32;
        stride[s] = 2ll * ld[s];
        row_ints += (size_t)stride[s];
    }
    if (nsp > 0) {
        size_t have = 0;
        bool grows = false;
        for (int s = 0; s < NS; s++) {
            have += ctx->sp[s].cap;
            grows |= ctx->sp[s].cap < (size_t)nsp * stride[s] * sizeof(int);
        }
        const size_t need = (size_t)nsp * row_ints * sizeof(int);
        if (grows) {
            // only when the buffers must grow: cudaMemGetInfo can take
            // milliseconds (it stalled repeated calls by up to 19 ms)
            size_t freeb = 0, totb = 0;
            cudaMemGetInfo(&freeb, &totb);
            if (need > (size_t)(0.8 * (double)(freeb + have))) {
                snprintf(ctx->errbuf, sizeof(ctx->errbuf), "special rows need %zu bytes on the device", need);
                return SW_ENOMEM;
            }
        }
        hck[2] = hnow();
        for (int s = 0; s < NS; s++) {
            if ((rc = grow(ctx, ctx->sp[s], (size_t)nsp * stride[s] * sizeof(int)))) return rc;
            if ((rc = grow_host(ctx, ctx->flags[s], nsp * sizeof(unsigned int), true))) return rc;
            memset(ctx->flags[s].p, 0, nsp * sizeof(unsigned int));
        }
        for (int s = 0; s < NS; s++) {
            if ((rc = grow_host(ctx, ctx->colp[s], (size_t)nb * sizeof(unsigned int), true))) return rc;
            memset(ctx->colp[s].p, 0, (size_t)nb * sizeof(unsigned int));
        }
        // staging window: every special row when they fit in ~1 GiB of pinned
        // memory (a one-wave matrix completes all its rows together), else as
        // many as fit (at least 2)
        const size_t row_bytes = (size_t)2 * (n + 64) * sizeof(int32_t);
        ctx->nstage = (int)std::max<size_t>(2, std::min<size_t>((size_t)nsp, ((size_t)1 << 30) / row_bytes));
        if ((rc = grow_host(ctx, ctx->stage, row_bytes * ctx->nstage, false))) return rc;
        while ((int)ctx->ev_row.size() < ctx->nstage) {
            cudaEvent_t ev;
            CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
            ctx->ev_row.push_back(ev);
        }
    }

    // With a caller stream, every kernel of the call is launched on it (so the
    // caller's CUDA events bracket them); otherwise on the library stream.
    cudaStream_t st = user_stream ? user_stream : ctx->stream;
    char *misc = (char *)ctx->misc.p;
    int *d_err = (int *)(misc + 0);
    int *d_gbest = (int *)(misc + 8);
    int *d_hit_band = (int *)(misc + 12);
    unsigned long long *d_hit_key = (unsigned long long *)(misc + 16);
    unsigned long long *d_replays = (unsigned long long *)(misc + 24);
    int4 *d_res = (int4 *)(misc + 32);
    int *d_tickets = (int *)(misc + 64);  // MAX_STRIPES

    hck[3] = hnow();
    CK(cudaEventRecord(ctx->ev[0], st));
    CK(cudaMemsetAsync(misc, 0, 16, st));
    CK(cudaMemsetAsync(d_hit_band, 0x7f, 4, st));
    CK(cudaMemsetAsync(d_hit_key, 0xff, 8, st));
    CK(cudaMemsetAsync(d_replays, 0, 8, st));
    CK(cudaMemsetAsync(d_tickets, 0, MAX_STRIPES * sizeof(int), st));
    for (int s = 0; s < NS; s++) CK(cudaMemsetAsync(ctx->progress[s].p, 0, (size_t)(nb + 1) * sizeof(int), st));
    {
        const long long words = wa + wb;
        const int tpb = 256;
        sw_encode_kernel<<<(unsigned)((words + tpb - 1) / tpb), tpb, 0, st>>>(
            J.dA, J.m, J.revA, (uint32_t *)ctx->a2.p, wa, J.dB, J.n, J.revB, (uint32_t *)ctx->b2.p, wb, d_err);
        CK(cudaGetLastError());
    }
    CK(cudaEventRecord(ctx->ev[1], st));
    hck[4] = hnow();

    FillArgs a{};
    a.m = m;
    a.n = n;
    a.nb = nb;
    a.go = J.go;
    a.ge = J.ge;
    a.gf = J.go + J.ge;
    a.one = 1;
    for (int x = 0; x < 4; x++) {
        uint32_t w = 0;
        for (int y = 0; y < 4; y++) {
            const int v = (x == y ? J.ma : J.mi) + a.gf;
            w |= (uint32_t)(uint8_t)(int8_t)v << (8 * y);
        }
        a.prof[x] = w;
    }
    a.A2 = (const uint32_t *)ctx->a2.p;
    a.B2 = (const uint32_t *)ctx->b2.p;
    a.err = d_err;
    a.k = (int)(nsp > 0 ? J.k : 0);
    a.gbest = d_gbest;
    a.slots = (int4 *)ctx->slots.p;
    a.goal = J.goal;
    a.hit_w = J.hit_w;
    a.anchor_gap = J.anchor_gap ? 1 : 0;
    a.match = J.match ? 1 : 0;
    a.mjc = (int)J.mjc;
    a.mH = J.mH;
    a.mF = J.mF;
    a.hit_key = d_hit_key;
    a.hit_band = d_hit_band;
    a.replays = d_replays;
    a.epoch = J.epoch;
    a.timeout_ns = ctx->timeout_ns;
    a.nstripes = NS;
    a.force_slow = 0;
    a.dbg = nullptr;
    if (getenv("SWB_DEBUG_TIMES")) {
        if ((rc = grow(ctx, ctx->dbg, (size_t)nb * 80 * sizeof(unsigned long long)))) return rc;
        CK(cudaMemsetAsync(ctx->dbg.p, 0, (size_t)nb * 80 * sizeof(unsigned long long), st));
        a.dbg = (unsigned long long *)ctx->dbg.p;
        ctx->dbg_n = nb;
    }
    for (int s = 0; s < NS; s++) {
        StripeArgs &S = a.st[s];
        S.col0 = (int)col0[s];
        S.w = (int)wid[s];
        S.ncols_pad = (int)((wid[s] + W - 1) / W) * W;
        S.NT = S.ncols_pad / W + (use16 ? 1 : V.skew_tiles);
        S.rowb = (int2 *)ctx->rowb[s].p;
        S.progress = (int *)ctx->progress[s].p;
        S.ticket = d_tickets + s;
        S.sp = nsp > 0 ? (int *)ctx->sp[s].p : nullptr;
        S.sp_stride = stride[s];
        S.sp_ld = ld[s];
        unsigned int *fd = nullptr;
        if (nsp > 0) CK(cudaHostGetDevicePointer((void **)&fd, ctx->flags[s].p, 0));
        S.row_done = fd;
        unsigned int *cp = nullptr;
        if (nsp > 0) CK(cudaHostGetDevicePointer((void **)&cp, ctx->colp[s].p, 0));
        S.colp = cp;
        if (J.rank_mode) {
            S.lb = J.c_lo > 0 ? ctx->recv.lb() : nullptr;
            S.lready = J.c_lo > 0 ? ctx->recv.lready() : nullptr;
            RecvArea right;
            right.base = ctx->right_base;
            right.rows = ctx->right_rows;
            S.rb = J.c_hi < n ? right.lb() : nullptr;
            S.rready = J.c_hi < n ? right.lready() : nullptr;
        } else {
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
    {
        void *args[] = {&a};
        const cudaError_t le = cudaLaunchKernel(fill_fn, dim3(grid), dim3(block), args, fill_smem, st);
        if (le != cudaSuccess) {
            cudaGetLastError();  // not sticky: do not fail the context's next call
            return cuda_fail(ctx, le, "cudaLaunchKernel(fill)");
        }
    }
    CK(cudaEventRecord(ctx->ev[2], st));
    sw_reduce_kernel<<<1, 256, 0, st>>>((const int4 *)ctx->slots.p, grid, J.local ? 1 : 0, d_hit_key, J.goal, d_res);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(ctx->res_h, d_res, sizeof(int4), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(ctx->res_h + 1, d_err, sizeof(int), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(ctx->res_h + 2, d_replays, sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    CK(cudaEventRecord(ctx->ev[3], st));

    // Stream special rows to the sink in ascending order while the fill runs.
    // A staged row is copied in column chunks as its band publishes final
    // columns (colp), and completed once every stripe has published the row
    // (row_done); the sink then runs on it in row order.
    int sink_rc = 0;
    long long bytes = 0;
    const int64_t nrow_out = J.rank_mode ? wid[0] : n;
    const int64_t sld = (NS == 1) ? ld[0] : nrow_out + 32;  // H at [0, sld), F at [sld, 2 sld)
    const int nstage = nsp > 0 ? ctx->nstage : 0;
    const int64_t CHUNK = 65536;  // columns per partial copy (512 KiB of H + F)
    std::vector<int64_t> copied((size_t)nstage * NS, 0);
    std::vector<char> sealed(nstage, 0);
    // SWB_DEBUG_HOST: host-side timeline of the special-row loop (stderr)
    const bool dbg_host = nsp > 0 && getenv("SWB_DEBUG_HOST") != nullptr;
    auto hms = [&]() { return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - h0).count(); };
    const double h_launch = hms();
    double h_fill = -1, h_sink_max = 0;
    long long n_copies = 0;
    auto row_ready = [&](long long q) -> bool {
        for (int s = 0; s < NS; s++)
            if (((volatile unsigned int *)ctx->flags[s].p)[q] == 0) return false;
        return true;
    };
    // copy what is final of staged row q; true when the row has been sealed
    auto pump = [&](long long q, bool &moved) -> int {
        const int slot = (int)(q % nstage);
        if (sealed[slot]) return SW_OK;
        const bool ready = row_ready(q);
        const int band = (int)(((q + 1) * J.k - 1) / BH);
        bool all = true;
        int32_t *dst = (int32_t *)ctx->stage.p + (size_t)slot * 2 * sld;
        for (int s = 0; s < NS; s++) {
            int64_t &c = copied[(size_t)slot * NS + s];
            int64_t avail = wid[s];
            if (!ready) avail = std::min<int64_t>(avail, ((volatile unsigned int *)ctx->colp[s].p)[band]);
            if (avail > c && (ready || avail - c >= CHUNK)) {
                const int32_t *src = (const int32_t *)ctx->sp[s].p + q * stride[s] + c;
                const int64_t off = (NS == 1 || J.rank_mode) ? 0 : col0[s];
                CK(cudaMemcpy2DAsync(dst + off + c, (size_t)sld * 4, src, (size_t)ld[s] * 4, (size_t)(avail - c) * 4, 2,
                                     cudaMemcpyDeviceToHost, ctx->side));
                n_copies++;
                c = avail;
                moved = true;
            }
            if (c < wid[s]) all = false;
        }
        if (ready && all) {
            CK(cudaEventRecord(ctx->ev_row[slot], ctx->side));
            sealed[slot] = 1;
            moved = true;
        }
        return SW_OK;
    };
    long long done = J.sink ? 0 : nsp;  // no sink (sw_align): the rows stay in HBM only
    while (done < nsp) {
        bool progress = false;
        if (dbg_host && h_fill < 0 && cudaEventQuery(ctx->ev[2]) == cudaSuccess) h_fill = hms();
        if (!sink_rc) {
            const long long hi = std::min<long long>(nsp, done + nstage);
            for (long long q = done; q < hi; q++)
                if ((rc = pump(q, progress))) return rc;
        }
        const int slot = (int)(done % nstage);
        if (sink_rc || sealed[slot]) {
            const cudaError_t qe = sink_rc ? cudaSuccess : cudaEventQuery(ctx->ev_row[slot]);
            if (qe == cudaSuccess) {
                if (!sink_rc) {
                    bytes += 8ll * nrow_out;
                    int32_t *row = (int32_t *)ctx->stage.p + (size_t)slot * 2 * sld;
                    const double t0 = dbg_host ? hms() : 0;
                    if (J.sink && J.sink(J.user, (done + 1) * J.k, row, row + sld, nrow_out)) sink_rc = SW_EABORTED;
                    if (dbg_host) h_sink_max = std::max(h_sink_max, hms() - t0);
                }
                sealed[slot] = 0;
                for (int s = 0; s < NS; s++) copied[(size_t)slot * NS + s] = 0;
                done++;
                progress = true;
            } else if (qe != cudaErrorNotReady) {
                return cuda_fail(ctx, qe, "special-row copy");
            }
        }
        if (!progress) {
            // nothing ready: make sure the fill is still running
            const cudaError_t fe = cudaEventQuery(ctx->ev[2]);
            if (fe == cudaSuccess && !sealed[slot] && !row_ready(done)) {
                CK(cudaStreamSynchronize(st));
                if (ctx->res_h[1].x == 1) return SW_EALPHABET;
                snprintf(ctx->errbuf, sizeof(ctx->errbuf), "special row %lld not published%s", done,
                         ctx->res_h[1].x == 2 ? " (kernel wait timeout)" : "");
                return SW_ECUDA;
            } else if (fe != cudaSuccess && fe != cudaErrorNotReady) {
                return cuda_fail(ctx, fe, "fill kernel");
            }
            std::this_thread::yield();
        }
    }
    if (dbg_host)
        fprintf(stderr, "[swb host] rows %lld copies %lld launched %.2f ms fill_seen %.2f ms loop_end %.2f ms max_sink %.3f ms nstage %d\n",
                nsp, n_copies, h_launch, h_fill, hms(), h_sink_max, nstage);
    if (sink_rc) CK(cudaStreamSynchronize(ctx->side));  // no copy may land in a reused staging slot later
    CK(cudaStreamSynchronize(st));
    if (dbg_host)
        fprintf(stderr, "[swb host] synced %.2f ms; pre-launch: variant %.2f grid %.2f meminfo %.2f staging %.2f encode %.2f\n", hms(),
                hck[0], hck[1], hck[2], hck[3], hck[4]);
    if (ctx->res_h[1].x == 1) return SW_EALPHABET;
    if (ctx->res_h[1].x == 2) {
        snprintf(ctx->errbuf, sizeof(ctx->errbuf), "fill kernel: border wait timeout (a neighbour stripe did not progress)");
        return SW_ECUDA;
    }
    if (sink_rc) return sink_rc;
    *res = ctx->res_h[0];

    float t01 = 0, t12 = 0, t23 = 0;
    cudaEventElapsedTime(&t01, ctx->ev[0], ctx->ev[1]);
    cudaEventElapsedTime(&t12, ctx->ev[1], ctx->ev[2]);
    cudaEventElapsedTime(&t23, ctx->ev[2], ctx->ev[3]);
    ctx->stats.encode_ms += t01;
    ctx->stats.fill_ms += t12;
    ctx->stats.reduce_ms += t23;
    ctx->stats.kernel_launches += 3;
    ctx->stats.replays += (long long)*(unsigned long long *)(ctx->res_h + 2);
    ctx->stats.special_rows += nsp;
    ctx->stats.special_bytes_d2h += bytes;
    ctx->stats.alpha = use16 ? -V.alpha : V.alpha;  // negative: packed 16x2 kernel
    ctx->stats.patched = patched ? 1 : 0;
    ctx->stats.warps = V.nw;
    ctx->stats.width = W;
    ctx->stats.grid = grid;
    if (J.local) {
        // Stage 2 can match against these rows while they stay resident
        S1Rows &R = ctx->s1;
        R.valid = NS == 1 && !J.rank_mode;
        R.m = J.m; R.n = J.n; R.k = J.k;
        R.ma = J.ma; R.mi = J.mi; R.go = J.go; R.ge = J.ge;
        R.ld = ld[0]; R.stride = stride[0];
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

extern "C" int sw_align_stage1_stripe(sw_ctx *ctx, const char *dseqA, int64_t m, const char *dseqB, int64_t n,
                                      int64_t c_lo, int64_t c_hi, int32_t epoch, int32_t match, int32_t mismatch,
                                      int32_t gap_open, int32_t gap_ext, int64_t special_row_interval,
                                      sw_row_sink sink, void *user, void *stream, sw_result *out)
{
    if (!valid_common(ctx, m, n, special_row_interval, sink, out)) return SW_EINVAL;
    if (!dseqA || !dseqB || m <= 0 || c_lo < 0 || c_hi > n || c_hi <= c_lo || epoch <= 0) return SW_EINVAL;
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
    // H, F of special row r at column j (row 0 and column 0: H = 0, F = -inf)
    auto fetch = [&](int64_t r, int64_t j, long long *h, long long *f) -> int {
        *h = 0;
        *f = NEG;
        if (r == 0 || j == 0) return SW_OK;
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
            J.mH = r > 0 ? sp + (r / k - 1) * R.stride : nullptr;
            J.mF = r > 0 ? J.mH + R.ld : nullptr;
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
                scr += (cta ? (MM_NWP + 3) : 3) * (Wd + 1);
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
            g.nparts = ncta;
            g.parts = (const MMPart *)ctx->mm_parts.p;
            g.res = (MMRes *)ctx->mm_res.p;
            sw_mm_split_cta_kernel<<<ncta, 32 * MM_NWP, 0, st>>>(g);
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
