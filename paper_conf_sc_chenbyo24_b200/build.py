"""Build the in-tree shared libraries with nvcc for sm_100a (no JIT, no torch extension).

    python -m paper_conf_sc_chenbyo24_b200.build          # libemb.so + synth/libsynth.so

The .so files land next to their sources so gpurun snapshots carry them to the GPU box.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
# no fast-math: FTZ / reassociation would break bit-exactness with the canonical oracle (C7)
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC", "-ftz=false", "-prec-div=true",
         "-prec-sqrt=true", "-fmad=false", "-Xptxas", "-v", "--expt-relaxed-constexpr"]

LIBS = {
    "emb": dict(srcs=[os.path.join(PKG, "csrc", "emb_runtime.cu")],
                deps=[os.path.join(PKG, "csrc", "emb_kernels.cuh"), os.path.join(ROOT, "include", "emb.h")],
                out=os.path.join(PKG, "libemb.so")),
    "synth": dict(srcs=[os.path.join(ROOT, "synth", "csrc", "synth_gen.cu")],
                  deps=[os.path.join(ROOT, "include", "synth.h")],
                  out=os.path.join(ROOT, "synth", "libsynth.so")),
}


def _stale(spec) -> bool:
    out = spec["out"]
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(s) > t for s in spec["srcs"] + spec["deps"] if os.path.exists(s))


def build(names=None, force: bool = False, verbose: bool = False) -> None:
    for name, spec in LIBS.items():
        if names and name not in names:
            continue
        if not force and not _stale(spec):
            continue
        cmd = [NVCC, *ARCH, *FLAGS, "-I", os.path.join(ROOT, "include"), *spec["srcs"], "-o", spec["out"] + ".tmp"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError(f"nvcc failed for {name}")
        os.replace(spec["out"] + ".tmp", spec["out"])
        log = os.path.join(os.path.dirname(spec["out"]), f".{name}_ptxas.log")
        with open(log, "w") as f:
            f.write(r.stderr)
        if verbose:
            sys.stdout.write(r.stderr)


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
