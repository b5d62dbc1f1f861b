"""CPU: the C-ABI libraries load and export every symbol their headers declare (no
compute calls -- there is no GPU here)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared(header):
    src = open(os.path.join(ROOT, "include", header)).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b((?:emb|synth)_[a-z0-9_]+)\s*\(", src)) - {"emb_allgather_fn"})


def _exported(so):
    out = subprocess.run(["nm", "-D", "--defined-only", so], capture_output=True, text=True).stdout
    return {l.split()[-1] for l in out.splitlines() if " T " in l}


def test_libemb_exports_every_declared_symbol():
    from paper_conf_sc_chenbyo24_b200 import _lib
    L = _lib.lib()
    decl = _declared("emb.h")
    assert "emb_forward" in decl and "emb_register_tables" in decl and len(decl) >= 14
    exp = _exported(_lib.LIB_PATH)
    for name in decl:
        assert name in exp, name
        assert hasattr(L, name)
        assert name in _lib.SIGNATURES, f"binding lacks {name}"
    assert set(_lib.SIGNATURES) <= set(decl)


def test_libsynth_exports_every_declared_symbol():
    import synth.gpu as g
    g.lib()
    exp = _exported(g._LIB_PATH)
    for name in _declared("synth.h"):
        assert name in exp, name


def test_no_gpu_fails_loudly():
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_sc_chenbyo24_b200 import emb as E
    with pytest.raises(E.EmbError) as ei:
        E.emb_init(0, 1, 0)
    assert ei.value.status == 3  # EMB_ERR_CUDA: no silent CPU fallback


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_sc_chenbyo24_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                s = open(os.path.join(dp, f)).read()
                imports = [l for l in s.splitlines() if re.match(r"\s*(from|import|#include)\s", l)]
                assert not any("oracle" in l for l in imports), f
    for dp, _, fs in os.walk(os.path.join(ROOT, "oracle")):
        for f in fs:
            if f.endswith(".py"):
                s = open(os.path.join(dp, f)).read()
                imports = [l for l in s.splitlines() if re.match(r"\s*(from|import)\s", l)]
                assert not any("paper_conf_sc_chenbyo24_b200" in l or "synth" in l for l in imports), f
