"""The two-build check that guards the immediate-patched packed kernels
(paper_conf_ipps_sandesm11_b200/patch_check.py), pinned on tiny kernels compiled here
(nvcc cross-compiles without a GPU): a magic constant used verbatim passes; a
constant derived from it (2*K folded into an immediate) is caught."""
import os
import shutil
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

SRC = r"""
#ifndef K
#define K 0x6b8b4567u
#endif
extern "C" __global__ void verbatim(unsigned *x) { x[threadIdx.x] = x[threadIdx.x] + K; }
#ifdef DERIVED
extern "C" __global__ void derived(unsigned *x) { x[threadIdx.x] = x[threadIdx.x] * 3u + 2u * K; }
#endif
"""


def _cubin(tmp_path, name, *flags):
    src = tmp_path / "k.cu"
    src.write_text(SRC)
    out = tmp_path / f"{name}.cubin"
    subprocess.run([NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-cubin", *flags, "-o", str(out), str(src)],
                   check=True, capture_output=True)
    return str(out)


@pytest.mark.skipif(shutil.which(NVCC) is None and not os.path.exists(NVCC), reason="nvcc not available")
def test_patch_check_accepts_verbatim_and_catches_derived(tmp_path):
    from paper_conf_ipps_sandesm11_b200 import patch_check

    alt = "-DK=0x1d2f3b61u"  # patch_check.MB[0], the alternative of MA[0]
    assert patch_check.main(_cubin(tmp_path, "a"), _cubin(tmp_path, "b", alt)) == 0
    assert patch_check.main(_cubin(tmp_path, "c", "-DDERIVED"), _cubin(tmp_path, "d", "-DDERIVED", alt)) == 1
