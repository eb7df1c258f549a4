"""SASS-level checks of the exact-arithmetic contract (reading R2, no FMA in
the predicate): no DFMA anywhere in libhdb; the f32-mode search kernels
contain no FFMA/FFMA2 (ptxas fuses mul.rn.f32x2 + add.rn.f32x2 otherwise);
the f64 filter kernels use FFMA2 (the filter is allowed to, its error bound
covers it); the exact-f64 kernels none.  CPU only (cuobjdump)."""
import os
import re
import shutil
import subprocess

import pytest

from paper_conf_ipps_gowanlockrblp17_b200 import LIB_PATH

CUOBJDUMP = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"


@pytest.fixture(scope="module")
def sass():
    if not os.path.exists(CUOBJDUMP):
        pytest.skip("cuobjdump not available")
    out = subprocess.run([CUOBJDUMP, "-sass", LIB_PATH], capture_output=True, text=True, check=True).stdout
    funcs = {}
    for chunk in re.split(r"\n\s*Function : ", out)[1:]:
        name, body = chunk.split("\n", 1)
        funcs[name.strip()] = body
    assert funcs
    return funcs


def _mode_kernels(sass, mode):
    """count kernel k_count<MODE> + recompute-write kernel k_search<MODE, true>"""
    return {k: v for k, v in sass.items() if re.search(rf"(k_countILi{mode}E|k_searchILi{mode}ELb1E)", k)}


def test_sm100a_code_present(sass):
    out = subprocess.run([CUOBJDUMP, "-lelf", LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_no_dfma_anywhere(sass):
    for name, body in sass.items():
        assert "DFMA" not in body, name


def test_f32_mode_has_no_ffma(sass):
    ks = _mode_kernels(sass, 0)
    assert len(ks) == 2
    for name, body in ks.items():
        assert "FFMA" not in body, name          # neither FFMA nor FFMA2
        assert "FMUL2" in body and "FADD2" in body, name


# every kernel that evaluates the predicate, by precision (template argument in the mangled name)
_F32_KERNELS = r"(k_countILi0E|k_searchILi0E|k_fusedILi0E|k_sparseILb0E|k_sample_countILb0E|k_paper_globalILb0E|k_paper_sharedILb0E|k_qlanesILi0E)"
_F64_EXACT_KERNELS = r"(k_countILi2E|k_searchILi2E|k_fusedILi2E|k_sparseILb1E|k_sample_countILb1E|k_paper_globalILb1E|k_paper_sharedILb1E)"


def test_every_f32_predicate_kernel_has_no_ffma(sass):
    """All f32-mode kernels (the default single pass k_fused<0>, the sparse
    thread-per-query kernels, the sampled count, the paper's two kernels, the
    query-lane single pass): fl(fl(dx^2) + fl(dy^2)) must never be contracted."""
    ks = {k: v for k, v in sass.items() if re.search(_F32_KERNELS, k)}
    assert len(ks) == 10, sorted(ks)   # (k_qlanes<0>: id and position output)
    for name, body in ks.items():
        assert "FFMA" not in body, name


def test_every_exact_f64_kernel_has_no_fma(sass):
    ks = {k: v for k, v in sass.items() if re.search(_F64_EXACT_KERNELS, k)}
    assert len(ks) == 8, sorted(ks)
    for name, body in ks.items():
        assert "FFMA" not in body and "DFMA" not in body and "DMUL" in body, name


def test_filter_and_exact_kernels(sass):
    filt = _mode_kernels(sass, 1)
    exact = _mode_kernels(sass, 2)
    assert len(filt) == 2 and len(exact) == 2
    for name, body in filt.items():
        assert "FFMA2" in body and "DMUL" in body, name   # f32 filter + exact f64 fallback
    for name, body in exact.items():
        assert "FFMA" not in body and "DMUL" in body, name
