"""Build libcof.so in-tree: nvcc for the sm_100a kernels, g++/OpenMP for the host side.

``python -m paper_conf_socc_jinv23_b200.build`` (or ``__graft_entry__.build()``).
The library links the CUDA runtime statically and needs only the driver at run time.
"""
from __future__ import annotations

import glob
import hashlib
import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(HERE, "libcof.so")
BUILD = os.path.join(HERE, "_build")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
VARIANT_SOURCES = {"single.cu", "finder.cu"}   # the sources a variant build's -D defines apply to


def _sources():
    cu = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    cpp = sorted(glob.glob(os.path.join(CSRC, "*.cpp")))
    hdr = sorted(glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh"))
                 + glob.glob(os.path.join(INCLUDE, "*.h")))
    return cu, cpp, hdr


def _digest(files):
    h = hashlib.sha256()
    for f in files:
        h.update(f.encode())
        with open(f, "rb") as fh:
            h.update(fh.read())
    return h.hexdigest()


def _local_includes(src, seen=None):
    """Local headers (csrc/, include/) that ``src`` includes, transitively."""
    import re
    seen = set() if seen is None else seen
    for name in re.findall(r'#include\s+"([^"]+)"', open(src).read()):
        for d in (os.path.dirname(src), CSRC, INCLUDE):
            path = os.path.join(d, name)
            if os.path.exists(path):
                if path not in seen:
                    seen.add(path)
                    _local_includes(path, seen)
                break
    return sorted(seen)


def _generate():
    gen = os.path.join(CSRC, "gen_csa.py")
    out = os.path.join(CSRC, "csa_gen.cuh")
    if not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(gen):
        text = subprocess.check_output([sys.executable, gen]).decode()
        with open(out, "w") as f:
            f.write(text)


def build(force: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """Build libcof.so (or, with ``defines`` such as "COF_SINGLE_SW=20", a variant library at
    ``out`` for A/B measurements, loaded through COF_LIB)."""
    _generate()
    cu, cpp, hdr = _sources()
    lib = out or LIB
    digest = _digest(cu + cpp + hdr + [__file__]) + "".join(defines)
    build_dir = BUILD if not defines else BUILD + "_" + "_".join(d.replace("=", "") for d in defines)
    stamp = os.path.join(build_dir, "stamp")
    if not force and os.path.exists(lib) and os.path.exists(stamp) and open(stamp).read() == digest:
        return lib
    os.makedirs(build_dir, exist_ok=True)
    dflags = [f"-D{d}" for d in defines]
    objs = []
    procs = []
    def compile_obj(src, cmd, obj):
        # per-object stamp: the source, the local headers it includes (transitively) and the
        # command; an unchanged object is not rebuilt
        d = _digest([src, *_local_includes(src)]) + " ".join(cmd)
        ostamp = obj + ".stamp"
        if not force and os.path.exists(obj) and os.path.exists(ostamp) and open(ostamp).read() == d:
            return
        procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT), ostamp, d))

    # a variant build (defines) recompiles only the sources the defines are for (VARIANT_SOURCES)
    # and shares every other object with the main build
    os.makedirs(BUILD, exist_ok=True)

    def where(src):
        if defines and os.path.basename(src) not in VARIANT_SOURCES:
            return BUILD, []
        return build_dir, dflags

    for src in cu:
        bdir, df = where(src)
        obj = os.path.join(bdir, os.path.basename(src) + ".o")
        cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-fopenmp",
               "-Xptxas", "-v" if verbose else "-O3", *df, "-I", INCLUDE, "-c", src, "-o", obj]
        compile_obj(src, cmd, obj)
        objs.append(obj)
    for src in cpp:
        bdir, df = where(src)
        obj = os.path.join(bdir, os.path.basename(src) + ".o")
        cmd = ["g++", "-O3", "-std=c++17", "-fPIC", "-fopenmp", "-Wall", *df, "-I", INCLUDE,
               "-I", os.path.join(CUDA, "include"), "-c", src, "-o", obj]
        compile_obj(src, cmd, obj)
        objs.append(obj)
    for cmd, p, ostamp, d in procs:
        out, _ = p.communicate()
        if p.returncode != 0:
            sys.stderr.write(out.decode(errors="replace"))
            raise RuntimeError("build failed: " + " ".join(cmd))
        if verbose and out:
            sys.stderr.write(out.decode(errors="replace"))
        with open(ostamp, "w") as f:
            f.write(d)
    tmp = lib + f".{os.getpid()}.tmp"
    cmd = ["g++", "-shared", "-fopenmp", "-o", tmp, *objs, "-L", os.path.join(CUDA, "lib64"),
           "-lcudart_static", "-ldl", "-lrt", "-lpthread", "-Wl,--no-undefined"]
    subprocess.check_call(cmd)
    os.replace(tmp, lib)
    with open(stamp, "w") as f:
        f.write(digest)
    return lib


if __name__ == "__main__":
    defs = [a[2:] for a in sys.argv[1:] if a.startswith("-D")]
    outs = [a[6:] for a in sys.argv[1:] if a.startswith("--out=")]
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, defines=defs, out=outs[0] if outs else None))
