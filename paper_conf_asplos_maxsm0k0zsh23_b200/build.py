"""Build libgzkp.so in-tree: nvcc for sm_100a only, one object per curve in
parallel, then one shared library.  No JIT cache: the .so travels with the repo
snapshot to the GPU box.

    python -m paper_conf_asplos_maxsm0k0zsh23_b200.build [--force] [--verbose]
"""

from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
BUILD = os.path.join(HERE, "_build")
LIB = os.path.join(HERE, "libgzkp.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-O2",
         "--expt-relaxed-constexpr", "-I", os.path.join(ROOT, "include"), "-I", CSRC]


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _headers():
    return sorted(glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h"))
                  + [os.path.join(ROOT, "include", "gzkp.h")])


def _newest(paths):
    return max(os.path.getmtime(p) for p in paths)


def _deps(obj: str, src: str):
    """Headers a TU includes, from the depfile nvcc wrote next to the object
    (all headers when there is none yet)."""
    dep = obj[:-2] + ".d"
    try:
        with open(dep) as f:
            text = f.read().replace("\\\n", " ")
        files = [w for w in text.split(":", 1)[1].split() if os.path.exists(w)]
        return files + [src]
    except (OSError, IndexError):
        return _headers() + [src]


def _compile(src: str, verbose: bool, build_dir: str = BUILD, defines=()) -> str:
    obj = os.path.join(build_dir, os.path.basename(src)[:-3] + ".o")
    cmd = [NVCC, *ARCH, *FLAGS, *[f"-D{d}" for d in defines], "-MD", "-MF", obj[:-2] + ".d", "-c", src, "-o", obj]
    if verbose:
        cmd += ["-Xptxas", "-v"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    if verbose and r.stderr:
        sys.stderr.write(r.stderr)
    return obj


def build(force: bool = False, verbose: bool = False, defines=(), lib: str = LIB) -> str:
    """Recompile each translation unit whose object is older than the source or
    any header in its depfile (headers edited while a build runs are caught:
    the check is per object, never "library newer than the sources"), then
    relink if any object is newer than the library."""
    srcs = _sources()
    build_dir = BUILD if not defines else BUILD + "_" + "_".join(d.replace("=", "") for d in defines)
    os.makedirs(build_dir, exist_ok=True)
    todo = []
    objs = []
    for s in srcs:
        obj = os.path.join(build_dir, os.path.basename(s)[:-3] + ".o")
        objs.append(obj)
        if force or verbose or not os.path.exists(obj) or os.path.getmtime(obj) < _newest(_deps(obj, s)):
            todo.append(s)
    if todo:
        with cf.ThreadPoolExecutor(max_workers=max(1, min(len(todo), os.cpu_count() or 4))) as ex:
            list(ex.map(lambda s: _compile(s, verbose, build_dir, defines), todo))
    if not todo and os.path.exists(lib) and os.path.getmtime(lib) >= _newest(objs):
        return lib
    tmp = lib + ".tmp.%d" % os.getpid()
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart", "-ldl"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    # experiment builds: python -m ...build -DGZKP_COOP_SOS=1 --out path/libgzkp_x.so
    defs = [a[2:] for a in sys.argv[1:] if a.startswith("-D")]
    out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else LIB
    print(build(force="--force" in sys.argv, verbose="--verbose" in sys.argv, defines=defs, lib=out))
