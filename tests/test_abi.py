"""C-ABI library checks that need no GPU (-m "not gpu")."""
import ctypes as C
import os
import re
import subprocess

import pytest

from paper_conf_cgo_xuwglgq14_b200 import build as B
from paper_conf_cgo_xuwglgq14_b200 import gstm as G

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def so():
    return B.build()


def header_functions():
    src = open(os.path.join(ROOT, "include", "gstm.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return set(re.findall(r"\b(gstm_[a-z_]+)\s*\(", src))


def test_header_declares_and_library_exports_every_symbol(so):
    declared = header_functions()
    assert len(declared) >= 25
    out = subprocess.check_output(["nm", "-D", "--defined-only", so], text=True)
    exported = set(re.findall(r" T (gstm_[a-z_]+)$", out, flags=re.M))
    assert declared == exported, (declared ^ exported)
    assert set(G.EXPORTS) == declared


def test_library_is_sm100a_and_self_contained(so):
    out = subprocess.check_output(["cuobjdump", "--list-elf", so], text=True)
    assert "sm_100a" in out
    deps = subprocess.check_output(["ldd", so], text=True)
    assert "libcudart" not in deps          # static cudart: nothing to resolve on the GPU box
    sass = subprocess.check_output(["cuobjdump", "-sass", so], text=True)
    funcs = dict(re.findall(r"Function : (\S+)\n(.*?)(?=\n\s*Function : |\Z)", sass, flags=re.S))
    split = funcs["_ZN4gstm10stm_kernelINS_6BankWLELi1ELb0ELi0EEEvNS_7KParamsE"]    # HV, paper layout
    paired = funcs["_ZN4gstm10stm_kernelINS_6BankWLELi1ELb1ELi0EEEvNS_7KParamsE"]   # HV, paired layout
    # the hot path is made of L2 atomics / strong gpu-scope accesses
    assert "ATOMG.E.OR.STRONG.GPU" in split and "LDG.E.STRONG.GPU" in split
    assert "ATOMG.E.OR.64.STRONG.GPU" in paired and "LDG.E.64.STRONG.GPU" in paired
    # one MEMBAR (the l.82 release fence) in the paper layout, none paired
    assert split.count("MEMBAR") == 1 and paired.count("MEMBAR") == 0
    # the bank kernels' logs stay in registers: no local-memory access at all
    # (a dynamically indexed log pass once moved them to a 128 B stack frame)
    for body in (split, paired):
        assert "LDL" not in body and "STL" not in body
    # the shared-memory log policy really uses shared memory: KM's
    # and RA's HV kernels keep their logs in LDS/STS (RA: no local memory at
    # all; KM keeps a few batch temporaries of its 17-word read on the stack)
    for wl in ("4KmWL", "4RaWL"):
        k = funcs[f"_ZN4gstm10stm_kernelINS_{wl}ELi1ELb0ELi0EEEvNS_7KParamsE"]
        assert k.count("LDS") >= 16 and k.count("STS") >= 16
    ra = funcs["_ZN4gstm10stm_kernelINS_4RaWLELi1ELb0ELi0EEEvNS_7KParamsE"]
    assert "LDL" not in ra and "STL" not in ra


def test_loads_and_host_only_calls(so):
    L = G.lib()
    assert L.gstm_api_version() == 2
    p = G.gstm_default_params("bank")
    assert p.n_words == 1 << 20 and p.block_threads == 256 and p.k_lock == 8
    # A3.l71's optional pre-lock VBV: on where it pays (KM 4x), off for HT
    assert [G.gstm_default_params(w).prelock_vbv for w in ("ra", "bank", "ht", "eb", "km")] == [1, 1, 0, 1, 1]
    # the adaptive contention manager: on for EB (its A > 16 kernels), off elsewhere
    assert [G.gstm_default_params(w).serial_after for w in ("ra", "bank", "ht", "eb", "km")] == [0, 0, 0, 4, 0]
    assert G.gstm_default_params("eb").serial_commits == 4
    # the gated pipelined lock round: k-means only
    assert [G.gstm_default_params(w).lock_pipeline_gated for w in ("ra", "bank", "ht", "eb", "km")] == [0, 0, 0, 0, 1]
    # EB's adaptive pipelined round
    e = G.gstm_default_params("eb")
    assert (e.lock_pipeline, e.pipeline_max_locks, e.pipeline_abort) == (16, 16, 100)
    assert [G.gstm_default_params(w).pipeline_abort for w in ("ra", "bank", "ht", "km")] == [0, 0, 0, 0]
    with pytest.raises(G.GstmError):
        G.gstm_default_params(9)


def test_create_fails_loudly_without_gpu(so):
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except ImportError:
        pass
    with pytest.raises(G.GstmError, match="no CUDA device"):
        G.Gstm(1024, 10)


def test_product_path_does_not_import_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_cgo_xuwglgq14_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", txt, flags=re.M), f
                assert "oracle/" not in txt.replace("oracle/gen.c", ""), f
