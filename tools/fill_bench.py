#!/usr/bin/env python3
"""Kernel-level timing of the Stage-1 fill (no reverse pass) for tuning:
python tools/fill_bench.py C3 [variants...] [--k K] [--reps R]."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402


def band_times(ctx):
    """Per-band timestamps (needs SWB_DEBUG_TIMES=1): returns an (nb, 4) array in us."""
    import ctypes

    import numpy as np

    lib = ctx._lib
    lib.swb_debug_times.restype = ctypes.c_int64
    buf = (ctypes.c_uint64 * (80 * 40000))()
    n = lib.swb_debug_times(ctx._h, buf, len(buf))
    raw = np.frombuffer(buf, dtype=np.uint64, count=n).reshape(-1, 80)
    for i in (0, 1, len(raw) // 2):
        print("   band", i, "replays", raw[i, 9], "thr/tmax per warp,unit:", [(int(x >> 32), int(x & 0xffffffff) - (1 << 32 if (x & 0xffffffff) >= (1 << 31) else 0)) for x in raw[i, 64:80]])
    a = raw[:, :64].astype(np.float64)
    a[:, 9] = 0
    t0 = a[a > 1e12].min()
    a = np.where(a > 0, (a - t0) / 1e3, np.nan)
    return a


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    opts = dict(a[2:].split("=") for a in sys.argv[1:] if a.startswith("--"))
    wl = args[0] if args else "C2"
    variants = [int(v) for v in args[1:]] or [-1]  # -1: the library's automatic choice
    reps = int(opts.get("reps", 2))
    if wl.startswith("R"):  # R<m>x<n>: random pair with one plant, e.g. R2000000x300000
        mm, nn = (int(x) for x in wl[1:].split("x"))
        k = int(opts.get("k", 0))
        A, B = synth.random_pair(99, mm, nn, plant_len=min(mm, nn) // 4, s=0.02, g=0.002)
    else:
        cfg = synth.CONFIGS[wl]
        k = int(opts.get("k", cfg.k))
        A, B = synth.make_pair(cfg)
    dA = torch.from_numpy(A).cuda()
    dB = torch.from_numpy(B).cuda()
    from paper_conf_ipps_sandesm11_b200 import Context

    for v in variants:
        if v >= 0:
            os.environ["SWB_VARIANT"] = str(v)
        else:
            os.environ.pop("SWB_VARIANT", None)
        ctx = Context(0)
        best = None
        for _ in range(reps):
            r, _ = ctx.align_stage1_dev(dA.data_ptr(), len(A), dB.data_ptr(), len(B), 1, -3, 3, 2, k=k,
                                        sink=(lambda *x: False) if k else None)
            st = ctx.stats()
            if best is None or st["fill_ms"] < best["fill_ms"]:
                best = st
        cells = len(A) * len(B)
        if os.environ.get("SWB_DEBUG_TIMES"):
            import numpy as np
            t = band_times(ctx)
            np.set_printoptions(linewidth=250, precision=1, suppress=True)
            print("  slots: 0 start | 1 first tile | 15 end (int32 kernel: 2-4 quarter intervals; packed: 2 tile-0 border ready, 3 upstream progress, 4 spins) | 5-7 border waits")
            for i in list(range(0, min(len(t), 3))) + [len(t) // 2]:
                print("   band", i, t[i][:16])
            lag = np.diff(t[:, 1])
            print(f"  start lag us mean={np.nanmean(lag):.1f} median={np.nanmedian(lag):.1f}; band dur us mean={np.nanmean(t[:,15]-t[:,1]):.0f}; "
                  f"first tile of the last band at {np.nanmax(t[:,1]):.0f} us, last band end {np.nanmax(t[:,15]):.0f} us")
        print(f"{wl} v{v} k={k} result={r.astuple()} fill_ms={best['fill_ms']:.2f} total_ms={best['total_ms']:.2f} "
              f"GCUPS(fill)={cells / best['fill_ms'] / 1e6:.1f} alpha={best['alpha']} warps={best['warps']} "
              f"grid={best['grid']} replays={best['replays']}", flush=True)
        ctx.close()


if __name__ == "__main__":
    main()

