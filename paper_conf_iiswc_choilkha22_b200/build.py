"""Build libsr_mha.so in-tree: nvcc for sm_100a, one object per .cu, linked into one shared library.

Usage: python -m paper_conf_iiswc_choilkha22_b200.build [--force] [--verbose]
       [--define NAME=VALUE ...] [--out PATH]   (experiment builds: extra -D flags, another .so; load
                                                  it with SR_MHA_LIB=PATH)
"""
from __future__ import annotations

import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libsr_mha.so")
BUILD = os.path.join(HERE, "_build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
SOURCES = ["abi.cu", "k_ir.cu", "k_simt_f32.cu", "k_g1.cu", "k_gemm2.cu", "k_softmax.cu", "k_sd.cu", "k_bwd.cu", "k_fused.cu", "k_conc.cu", "tc_host.cu", "k_sched.cu"]
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall", "--expt-relaxed-constexpr",
         "-I", os.path.join(ROOT, "include"), "-I", CSRC]


def _deps():
    files = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(ROOT, "include", "sr_mha.h")]
    return max(os.path.getmtime(f) for f in files)


def build(force: bool = False, verbose: bool = False, defines=(), out: str = LIB) -> str:
    if not force and not defines and os.path.exists(out) and os.path.getmtime(out) >= _deps():
        return out
    bdir = BUILD if not defines else os.path.join(BUILD, "x_" + "_".join(d.replace("=", "") for d in defines))
    os.makedirs(bdir, exist_ok=True)
    extra = (["-Xptxas", "-v"] if verbose else []) + [f"-D{d}" for d in defines]

    def compile_one(src):
        obj = os.path.join(bdir, src.replace(".cu", ".o"))
        cmd = [NVCC, *FLAGS, *extra, "-c", os.path.join(CSRC, src), "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
        if verbose:
            sys.stderr.write(r.stderr)
        return obj

    with ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        objs = list(ex.map(compile_one, SOURCES))
    tmp = out + f".tmp{os.getpid()}"
    cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp, *objs]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, out)
    return out


if __name__ == "__main__":
    a = sys.argv[1:]
    defs = [a[i + 1] for i, x in enumerate(a) if x == "--define"]
    o = next((a[i + 1] for i, x in enumerate(a) if x == "--out"), LIB)
    print(build(force="--force" in a, verbose="--verbose" in a, defines=defs, out=os.path.abspath(o)))
