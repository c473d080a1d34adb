"""Build libarlo.so in-tree with nvcc for sm_100a (B200) only.

    python -m paper_conf_icpp_tanlyl024_b200.build [--verbose-ptxas]
    python -m paper_conf_icpp_tanlyl024_b200.build --variant NAME -DMACRO=V ...   (A/B experiments:
        build/libarlo_NAME.so with extra defines, loaded when ARLO_LIB_VARIANT=NAME)

Each translation unit under csrc/ is compiled to an object with
``-gencode arch=compute_100a,code=sm_100a -lineinfo -O3`` (in parallel), then
linked into ``paper_conf_icpp_tanlyl024_b200/libarlo.so`` against the static
CUDA runtime (no link-time libcuda dependency: the TMA encoder is resolved at
run time through cudaGetDriverEntryPoint, so the library also loads on a
GPU-less host for the export checks).
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libarlo.so")
SOURCES = ["embed_ln.cu", "gemm_simt.cu", "gemm_tc.cu", "gemm_splitk.cu", "encoder_fused.cu", "attention.cu", "head.cu", "runtime.cu", "sched.cpp"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nvcc() -> str:
    p = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
    if not os.path.exists(p):
        raise RuntimeError("nvcc not found")
    return p


def _compile(src: str, verbose_ptxas: bool, defines=(), tag="") -> tuple:
    obj = os.path.join(BUILD, os.path.basename(src) + tag + ".o")
    cmd = [nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3", *defines,
           "-I", os.path.join(ROOT, "include"), "-c", os.path.join(CSRC, src), "-o", obj]
    if src.endswith(".cu"):
        cmd += ["--expt-relaxed-constexpr"]
        if verbose_ptxas:
            cmd += ["-Xptxas", "-v"]
    else:
        cmd = [nvcc(), "-x", "c++", "-O3", "-std=c++17", "-Xcompiler", "-fPIC,-O3",
               "-I", os.path.join(ROOT, "include"), "-c", os.path.join(CSRC, src), "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    return src, obj, r.returncode, r.stdout + r.stderr


def _stale(obj: str, src: str) -> bool:
    if not os.path.exists(obj):
        return True
    deps = [os.path.join(CSRC, src)] + [os.path.join(CSRC, f) for f in os.listdir(CSRC)
                                        if f.endswith((".h", ".cuh"))]
    deps += [os.path.join(ROOT, "include", f) for f in os.listdir(os.path.join(ROOT, "include"))]
    t = os.path.getmtime(obj)
    return any(os.path.getmtime(d) > t for d in deps)


def build(verbose_ptxas: bool = False, force: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    todo = [s for s in SOURCES if force or verbose_ptxas or _stale(os.path.join(BUILD, s + ".o"), s)]
    logs = []
    if todo:
        with cf.ThreadPoolExecutor(max_workers=min(8, len(todo))) as ex:
            for src, obj, rc, out in ex.map(lambda s: _compile(s, verbose_ptxas), todo):
                if out.strip():
                    logs.append(f"--- {src}\n{out}")
                if rc != 0:
                    raise RuntimeError(f"nvcc failed on {src}:\n{out}")
    objs = [os.path.join(BUILD, s + ".o") for s in SOURCES]
    if todo or not os.path.exists(LIB):
        cmd = [nvcc(), *ARCH, "-shared", "-o", LIB, *objs, "-cudart", "static", "-lpthread", "-ldl", "-lrt"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stdout}{r.stderr}")
    if verbose_ptxas:
        print("\n".join(logs))
    return LIB


def build_variant(name: str, defines) -> str:
    """Compile every source with extra -D flags into build/libarlo_<name>.so (A/B runs)."""
    os.makedirs(BUILD, exist_ok=True)
    tag = "." + name
    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        for src, obj, rc, out in ex.map(lambda s: _compile(s, False, defines, tag), SOURCES):
            if rc != 0:
                raise RuntimeError(f"nvcc failed on {src}:\n{out}")
    lib = os.path.join(BUILD, f"libarlo_{name}.so")
    objs = [os.path.join(BUILD, s + tag + ".o") for s in SOURCES]
    cmd = [nvcc(), *ARCH, "-shared", "-o", lib, *objs, "-cudart", "static", "-lpthread", "-ldl", "-lrt"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}{r.stderr}")
    return lib


if __name__ == "__main__":
    if "--variant" in sys.argv:
        name = sys.argv[sys.argv.index("--variant") + 1]
        print(build_variant(name, [a for a in sys.argv[1:] if a.startswith("-D")]))
    else:
        print(build(verbose_ptxas="--verbose-ptxas" in sys.argv, force="--force" in sys.argv))
