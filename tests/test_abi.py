"""CPU checks of the C-ABI boundary: libadainf.so loads without a GPU, exports every symbol the headers
declare, and compute calls fail loudly (no CPU fallback) when no sm_100 device is present."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_sigcomm_shubhas23_b200", "libadainf.so")


def declared_symbols():
    names = set()
    for h in ("adainf.h", "adainf_debug.h", "adainf_sched.h"):
        txt = open(os.path.join(ROOT, "include", h)).read()
        names |= set(re.findall(r"\b(adainf_[a-z0-9_]+)\s*\(", txt))
    return names


def test_library_loads_and_exports_all_declared_symbols():
    assert os.path.exists(LIB), "run __graft_entry__.build() first"
    L = ctypes.CDLL(LIB)
    missing = [s for s in sorted(declared_symbols()) if not hasattr(L, s)]
    assert not missing, missing
    assert len(declared_symbols()) >= 20


def test_no_cpu_fallback_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_sigcomm_shubhas23_b200 import binding as B
    from paper_conf_sigcomm_shubhas23_b200 import specs as S
    with pytest.raises(B.AdaInfError) as ei:
        B.Model(S.tiny_cnn_ee(), 4)
    assert ei.value.code == B.ERR_UNSUPPORTED


def test_product_package_never_imports_oracle():
    """The product path (package + bench hot path) must not route through the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_sigcomm_shubhas23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f), errors="ignore").read()
                assert "import oracle" not in txt and "oracle.h" not in txt and "from oracle" not in txt, f
