"""The benchmark and parity workloads are pure functions of their seeds
(synth/): pin every config's sequences by sha256 so a
numpy or generator change cannot silently change what bench.py times or what
the large-config parity tests check (SURVEY.md 8(d) "Each generated pair is
hashed (sha256) in the tests").  The shapes mirror Table II."""
import numpy as np
import pytest

import synth

GOLDEN = {
    "C1": "78e05abcb0960140c3b94121efcb7709b82caaba41c3601bb761733c4820375e",
    "C2": "8191f4e3fe4b5968407a92b0218b699a74bcfbbacd48f2ae332d41455e8f7de7",
    "C3": "d76da59d63555fb7ac65c2e38a0df08b8ae886c24fe69356638191fbe618cf9c",
    "C4": "5655a0008fce26b2d8eecc72d026f7936a71ad431758a4899b11905a2b3cfa71",
    "C5": "653de1365bc86d1e108b5d09c3e7813b0bb5fc4c5d49bc2e80c7e16f234b362c",
}
# Table II real sizes that C2 and C5 reproduce exactly
SIZES = {"C1": (50_000, 50_000), "C2": (542_868, 536_165), "C3": (5_000_000, 5_000_000),
         "C4": (10_000_000, 10_000_000), "C5": (32_799_110, 46_944_323)}


@pytest.mark.parametrize("name", sorted(GOLDEN))
def test_config_sha256(name):
    A, B = synth.make_pair(name)
    assert (len(A), len(B)) == SIZES[name]
    assert set(np.unique(A)) <= set(b"ACGT") and set(np.unique(B)) <= set(b"ACGT")
    assert synth.sha256_pair(A, B) == GOLDEN[name]


def test_c2_planted_segment():
    """C2 plants Table III row 2's shape: 92 gapless columns with 11
    substitutions from A[a0:] into B[b0:]."""
    cfg = synth.CONFIGS["C2"]
    A, B = synth.make_pair(cfg)
    a0, b0, L = cfg.params["a0"], cfg.params["b0"], cfg.params["L"]
    assert int((A[a0:a0 + L] != B[b0:b0 + L]).sum()) == cfg.params["n_sub"]
