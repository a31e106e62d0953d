"""SASS evidence for the design choices, read from the built library with cuobjdump (no GPU needed):

* the tensor-core chains (RDG stage 1 + BVS stage 2, §III-B/§III-D) are
  DMMA.8x8x4 and contain no warp shuffle: Butterfly Vector Swapping reuses the accumulator layout as the
  next MMA's A fragment; the no-BVS ablation instantiation does shuffle (so the check can fail);
* tiles arrive by TMA (UTMALDG) in the TMA instantiations of the stream and chain kernels;
* the CUDA-core engine issues DFMA/DADD/DMUL only (no DMMA), DESIGN.md §5.
"""
import os
import re
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_sc_zhanglyczcy24_b200", "liblora_stencil.so")


@pytest.fixture(scope="module")
def sass():
    tool = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(tool) or not os.path.exists(LIB):
        pytest.skip("cuobjdump or the built library is missing")
    txt = subprocess.run([tool, "-sass", LIB], capture_output=True, text=True, timeout=600).stdout
    funcs = {}
    for part in txt.split("Function : ")[1:]:
        name, _, body = part.partition("\n")
        funcs[name.strip()] = body
    assert funcs, "no kernels found in the library"
    return funcs


def _ops(body):
    return re.findall(r"/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Za-z0-9_.]*)", body)


def _pick(funcs, pattern):
    out = {n: b for n, b in funcs.items() if re.search(pattern, n)}
    assert out, pattern
    return out


def test_tc_chains_are_dmma_without_shuffles(sass):
    # tc2d_kernel<R, TMA, NOBVS=false> and tc3d_kernel<1, TMA>
    chains = {**_pick(sass, r"tc2d_kernelILi\dELb[01]ELb0E"), **_pick(sass, r"tc3d_kernelILi1ELb[01]E")}
    for name, body in chains.items():
        ops = _ops(body)
        assert any(o.startswith("DMMA.8x8x4") for o in ops), name
        assert not any(o.startswith("SHFL") for o in ops), name


def test_no_bvs_ablation_shuffles(sass):
    for name, body in _pick(sass, r"tc2d_kernelILi\dELb[01]ELb1E").items():
        assert any(o.startswith("SHFL") for o in _ops(body)), name


def test_tma_staging(sass):
    for pat in (r"tc2d_kernelILi\dELb1ELb0E", r"tc3d_kernelILi1ELb1E", r"rdg2d_kernelILi\dELi\dELi\dELb1E",
                r"rdg3df_kernel.*ELi\dELb1ELb[01]E"):
        for name, body in _pick(sass, pat).items():
            assert any(o.startswith("UTMALDG") for o in _ops(body)), name


def test_cuda_core_engine_has_no_dmma(sass):
    for name, body in _pick(sass, r"rdg2d_kernel|rdg3df_kernel").items():
        ops = _ops(body)
        assert any(o.startswith("DFMA") for o in ops), name
        assert not any(o.startswith("DMMA") for o in ops), name


def test_stencil_weights_in_uniform_registers(sass):
    # DESIGN.md §6 "Uniform-register weights": every DFMA of the fused 2D row-pair / PMA / star kernels
    # (single-GPU AND device-initiated-exchange instantiations) and of the fused 3D kernel takes its
    # weight from a uniform register (DFMA R, R, URx, R); a lane-0-only spin loop in the kernel made
    # ptxas keep the weights in vector registers (364 vs 429 GS/s on Box-2D49P)
    pats = (r"rdg2d_kernelILi\dELi[014]ELi[234]ELb[01]ELb[01]E", r"rdg3df_kernel.*ELi2ELb1ELb[01]E")
    for pat in pats:
        for name, body in _pick(sass, pat).items():
            dfma = [ln for ln in body.splitlines() if re.search(r"\bDFMA\b", ln)]
            assert dfma, name
            vec = [ln for ln in dfma if not re.search(r"\bUR\d+", ln)]
            assert len(vec) <= len(dfma) // 50, (name, len(vec), len(dfma), vec[:3])
