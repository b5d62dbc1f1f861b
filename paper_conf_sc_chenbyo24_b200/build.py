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
         "-prec-sqrt=true", "-fmad=false", "-Xptxas", "-v", "--expt-relaxed-constexpr",
         "--compress-mode=size"]   # compressed fatbin: the .so shrinks ~8x, loads the same SASS

CSRC = os.path.join(PKG, "csrc")
# the fused forward is instantiated per (weight, output) dtype pair: one source, four objects
_PAIRS = [("f32_f32", "float", "float"), ("f32_bf16", "float", "__nv_bfloat16"),
          ("bf16_f32", "__nv_bfloat16", "float"), ("bf16_bf16", "__nv_bfloat16", "__nv_bfloat16")]
LIBS = {
    "emb": dict(srcs=[os.path.join(CSRC, "emb_runtime.cu")] +
                     [(os.path.join(CSRC, "emb_inst.cu"), f"inst_{tag}",
                       [f"-DEMB_INST_WT={w}", f"-DEMB_INST_OT={o}", f"-DEMB_INST_NAME=pick_fwd_{tag}"])
                      for tag, w, o in _PAIRS],
                deps=[os.path.join(CSRC, f) for f in ("emb_kernels.cuh", "emb_dispatch.h", "emb_bwd.cuh",
                                                      "emb_bwd_sort.cuh", "emb_inst.cu")] +
                     [os.path.join(ROOT, "include", "emb.h")],
                out=os.path.join(PKG, "libemb.so")),
    "synth": dict(srcs=[os.path.join(ROOT, "synth", "csrc", "synth_gen.cu")],
                  deps=[os.path.join(ROOT, "include", "synth.h")],
                  out=os.path.join(ROOT, "synth", "libsynth.so")),
}


def _src(entry):
    """(path, object stem, extra flags) of a source entry (a path or such a tuple)."""
    if isinstance(entry, tuple):
        return entry
    return entry, os.path.basename(entry), []


def _stale(spec) -> bool:
    out = spec["out"]
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    paths = [_src(e)[0] for e in spec["srcs"]] + spec["deps"]
    return any(os.path.getmtime(p) > t for p in paths if os.path.exists(p))


def _nvcc(args):
    r = subprocess.run([NVCC, *args], capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed: " + " ".join(args[-3:]))
    return r.stderr


def build(names=None, force: bool = False, verbose: bool = False) -> None:
    """Compile every translation unit to an object in parallel, then link the .so."""
    for name, spec in LIBS.items():
        if names and name not in names:
            continue
        _build_one(name, spec, force, verbose)


def _build_one(name, spec, force, verbose, extra=()):
    from concurrent.futures import ThreadPoolExecutor
    if True:
        if not force and not _stale(spec):
            return
        objdir = os.path.join(os.path.dirname(spec["out"]), ".obj")
        os.makedirs(objdir, exist_ok=True)
        comp = [f for f in FLAGS if f != "-shared"] + list(extra)
        jobs = []
        for entry in spec["srcs"]:
            src, stem, defs = _src(entry)
            obj = os.path.join(objdir, stem + ".o")
            jobs.append((obj, [*ARCH, *comp, *defs, "-I", os.path.join(ROOT, "include"), "-c", src, "-o", obj]))
        with ThreadPoolExecutor(max_workers=min(len(jobs), os.cpu_count() or 4)) as ex:
            logs = list(ex.map(lambda j: _nvcc(j[1]), jobs))
        _nvcc([*ARCH, "-shared", "-Xcompiler", "-fPIC", *[j[0] for j in jobs], "-o", spec["out"] + ".tmp"])
        os.replace(spec["out"] + ".tmp", spec["out"])
        log = os.path.join(os.path.dirname(spec["out"]), f".{name}_ptxas.log")
        with open(log, "w") as f:
            f.write("".join(logs))
        if verbose:
            sys.stdout.write("".join(logs))


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
