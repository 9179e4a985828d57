"""Build libcudalign_b200.so in-tree for sm_100a (nvcc cross-compiles without a GPU).

    python -m paper_conf_ipps_sandesm11_b200.build [--force]
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libcudalign_b200.so")
SOURCES = [os.path.join(HERE, "csrc", "sw_api.cu")]
# The packed kernels with magic immediates (csrc/sw_fill16_patch.cu), embedded
# in the library and patched per scoring at run time.
PATCH_SRC = os.path.join(HERE, "csrc", "sw_fill16_patch.cu")
PATCH_CUBIN = os.path.join(HERE, "sw_fill16_patch.cubin")
MAGIC = {"NGE2": 0x6B8B4567, "NGF2": 0x327B23C6, "NGE16": 0x643C9869, "NGF16": 0x66334873,
         "NGE1": 0x2AE8944A, "NGF1": 0x625558EC}
# the alternative set of the two-build check (same order)
ALT_MAGIC = [0x1D2F3B61, 0x5E3A9B27, 0x49C1F6B3, 0x7A2D4E19, 0x3F6B2D85, 0x0B7E5C93]
import glob

DEPS = sorted(glob.glob(os.path.join(HERE, "csrc", "*"))) + [os.path.join(ROOT, "include", "cudalign_b200.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-shared",
]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in DEPS)


def check_patch_sites(path: str, required=("NGE2", "NGE16", "NGF16")) -> dict:
    """Every occurrence of a magic word in the cubin must be a 32-bit
    instruction immediate (byte 4 of a 16-byte SASS instruction); the loader
    (sw_api.cu patch_sites) refuses to patch otherwise."""
    import struct

    from . import patch_check

    data = open(path, "rb").read()
    text = patch_check.text_ranges(data)
    counts = {}
    for name, v in MAGIC.items():
        pat = struct.pack("<I", v)
        offs, i = [], data.find(pat)
        while i >= 0:
            offs.append(i)
            i = data.find(pat, i + 1)
        # inside a kernel's .text section, at byte 4 of a 16-byte instruction (the
        # 32-bit immediate field), counted from the section start
        sec = [next(((lo, hi) for lo, hi in text if lo <= o < hi), None) for o in offs]
        bad = [o for o, r in zip(offs, sec) if r is None or (o - r[0]) % 16 != 4]
        if bad:
            raise RuntimeError(f"{path}: magic {name} outside an instruction immediate at offsets {bad[:4]}")
        # ptxas must use the constant as written: a negated copy (x - (-K)) could not be patched
        if data.find(struct.pack("<I", (-v) & 0xFFFFFFFF)) >= 0:
            raise RuntimeError(f"{path}: the negation of magic {name} occurs (an unpatchable form)")
        counts[name] = len(offs)
    for name in required:
        if counts[name] == 0:
            raise RuntimeError(f"{path}: magic {name} not found (ptxas folded it?)")
    return counts


def build(force: bool = False, verbose: bool = False, defs: list | None = None, out_dir: str | None = None) -> str:
    """Build the library.  ``defs`` (extra -D flags) and ``out_dir`` (where the
    library and its cubin go) serve A/B experiments (tools/build_variant.py);
    the product build uses neither."""
    global LIB, PATCH_CUBIN
    if out_dir:
        os.makedirs(out_dir, exist_ok=True)
        LIB = os.path.join(out_dir, "libcudalign_b200.so")
        PATCH_CUBIN = os.path.join(out_dir, "sw_fill16_patch.cubin")
        force = True
    if not force and not stale():
        return LIB
    defs = list(defs or [])
    # in parallel: the patchable cubin twice (the magic set used at run time and
    # an alternative set; the SASS must agree up to the magic words,
    # patch_check.py) and the library's object; then the embedding object and the link
    ptmp = PATCH_CUBIN + f".tmp{os.getpid()}"
    palt = PATCH_CUBIN + f".alt{os.getpid()}"
    obj = LIB[:-3] + f".{os.getpid()}.o"  # nvcc picks the input kind by extension
    cflags = [f for f in FLAGS if f not in ("-Xcompiler", "-fPIC", "-shared")] + defs
    alt = [f"-DSWB_K_{k}={v:#x}u" for k, v in zip(MAGIC, ALT_MAGIC)]
    ocmd = [NVCC, *cflags, "-Xcompiler", "-fPIC", "-DSWB_PATCH_EXTERN", "-c", "-o", obj, *SOURCES]
    if verbose:
        ocmd.insert(1, "-Xptxas=-v")
        print(" ".join(ocmd))
    procs = [subprocess.Popen([NVCC, *cflags, "-cubin", "-o", ptmp, PATCH_SRC]),
             subprocess.Popen([NVCC, *cflags, *alt, "-cubin", "-o", palt, PATCH_SRC]),
             subprocess.Popen(ocmd)]
    if any([p.wait() for p in procs]):
        raise RuntimeError("nvcc failed")
    check_patch_sites(ptmp, ("NGE2", "NGE16", "NGF16") if not defs else ("NGE2",))
    from . import patch_check

    if patch_check.main(ptmp, palt):
        raise RuntimeError("patchable cubin: SASS depends on the magic values (a derived constant)")
    os.remove(palt)
    os.replace(ptmp, PATCH_CUBIN)
    emb_s = LIB[:-3] + f".embed{os.getpid()}.S"
    emb_o = emb_s[:-2] + ".o"
    with open(emb_s, "w") as f:
        f.write(".section .rodata\n.balign 16\n.globl swb_patch_cubin_begin\n.globl swb_patch_cubin_end\n"
                f"swb_patch_cubin_begin:\n.incbin \"{PATCH_CUBIN}\"\nswb_patch_cubin_end:\n"
                ".section .note.GNU-stack,\"\",@progbits\n")
    subprocess.check_call(["gcc", "-c", "-fPIC", "-o", emb_o, emb_s])
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp, obj, emb_o])
    for f in (obj, emb_s, emb_o):
        os.remove(f)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
