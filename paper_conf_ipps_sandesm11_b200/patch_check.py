#!/usr/bin/env python3
"""Check that a patchable cubin uses its magic immediates only verbatim:
disassemble two builds made with different magic sets, replace each magic by a
token, and compare the instruction streams per function.  A derived constant
(e.g. 2*K, K1+K2, -K) makes the streams differ.
python -m paper_conf_ipps_sandesm11_b200.patch_check a.cubin b.cubin

Also: text_ranges(data), the [start, end) file ranges of the ELF .text.*
sections (kernel code) of a cubin -- the only places a magic may be patched."""
import os
import re
import struct
import subprocess
import sys

MA = [0x6B8B4567, 0x327B23C6, 0x643C9869, 0x66334873, 0x2AE8944A, 0x625558EC]
MB = [0x1D2F3B61, 0x5E3A9B27, 0x49C1F6B3, 0x7A2D4E19, 0x3F6B2D85, 0x0B7E5C93]


def cuobjdump() -> str:
    """cuobjdump next to the nvcc the build uses (NVCC), else CUOBJDUMP, else PATH."""
    if os.environ.get("CUOBJDUMP"):
        return os.environ["CUOBJDUMP"]
    nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
    cand = os.path.join(os.path.dirname(nvcc), "cuobjdump")
    return cand if os.path.exists(cand) else "cuobjdump"


def text_ranges(data: bytes):
    """File ranges of the SHT_PROGBITS sections named .text.* of an ELF64 image."""
    if data[:4] != b"\x7fELF" or data[4] != 2:
        raise ValueError("not an ELF64 image")
    shoff = struct.unpack_from("<Q", data, 0x28)[0]
    shentsize, shnum, shstrndx = struct.unpack_from("<HHH", data, 0x3A)
    hdr = [struct.unpack_from("<IIQQQQ", data, shoff + i * shentsize) for i in range(shnum)]
    stroff = hdr[shstrndx][4]
    out = []
    for name, typ, _flags, _addr, off, size in hdr:
        nm = data[stroff + name: data.index(b"\0", stroff + name)].decode()
        if typ == 1 and nm.startswith(".text."):
            out.append((off, off + size))
    return out


def stream(path, magics):
    out = subprocess.run([cuobjdump(), "-sass", path], capture_output=True, text=True, check=True).stdout
    funcs, cur = {}, None
    for ln in out.splitlines():
        m = re.match(r"\s*Function : (\S+)", ln)
        if m:
            cur = m.group(1); funcs[cur] = []
            continue
        m = re.search(r"/\*[0-9a-f]{4,}\*/\s+(.*?);", ln)
        if m and cur:
            ins = m.group(1)
            for k, v in enumerate(magics):
                ins = re.sub(r"\b0x%x\b" % v, f"MAGIC{k}", ins)
            funcs[cur].append(ins)
    return funcs


def main(a, b):
    fa, fb = stream(a, MA), stream(b, MB)
    bad = 0
    for name in sorted(set(fa) | set(fb)):
        sa, sb = fa.get(name, []), fb.get(name, [])
        if sa != sb:
            bad += 1
            n = next((i for i, (x, y) in enumerate(zip(sa, sb)) if x != y), min(len(sa), len(sb)))
            print(f"DIFF {name}: {len(sa)} vs {len(sb)} instrs, first at {n}: {sa[n:n+1]} | {sb[n:n+1]}")
    print(f"{len(fa)} functions, {bad} differ")
    return bad


if __name__ == "__main__":
    sys.exit(1 if main(sys.argv[1], sys.argv[2]) else 0)
