"""Build libxreduce.so in-tree (nvcc, sm_100a only).

Usage: python tools/build_native.py [--force] [--ptxas-v]
The .so lands in paper_conf_ppopp_xutycc14_b200/ so it travels with gpurun
snapshots.  This file deliberately lives OUTSIDE the package: importing the
package loads the .so, which must not be required to build it.
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HERE = os.path.join(ROOT, "paper_conf_ppopp_xutycc14_b200")
CSRC = os.path.join(HERE, "csrc")
OBJ = os.path.join(HERE, "build")
SO = os.path.join(HERE, "libxreduce.so")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_dir() -> str:
    try:
        import nvidia.nccl  # type: ignore
        d = list(nvidia.nccl.__path__)[0]
        if os.path.exists(os.path.join(d, "include", "nccl.h")):
            return d
    except Exception:
        pass
    d = "/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl"
    return d


def _sources():
    cu = sorted(f for f in os.listdir(CSRC) if f.endswith(".cu"))
    cpp = sorted(f for f in os.listdir(CSRC) if f.endswith(".cpp"))
    hdr = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))]
    inc = os.path.join(ROOT, "include")
    hdr += [os.path.join(inc, f) for f in os.listdir(inc)]
    return cu, cpp, hdr


def _stale(obj: str, deps) -> bool:
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, ptxas_verbose: bool = False, quiet: bool = True,
          defines=(), so_path: str | None = None, obj_dir: str | None = None) -> str:
    """defines / so_path / obj_dir: A/B variants (tools/build_native.py --variant)."""
    OBJ = obj_dir or globals()["OBJ"]
    SO = so_path or globals()["SO"]
    os.makedirs(OBJ, exist_ok=True)
    nccl = _nccl_dir()
    inc = ["-I", os.path.join(ROOT, "include"), "-I", CSRC, "-I", os.path.join(nccl, "include")]
    cu, cpp, hdr = _sources()
    jobs = []
    objs = []
    for f in cu:
        src = os.path.join(CSRC, f)
        obj = os.path.join(OBJ, f + ".o")
        objs.append(obj)
        if force or _stale(obj, [src] + hdr):
            cmd = [NVCC, *ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC",
                   "--expt-relaxed-constexpr", *["-D" + d for d in defines], "-c", src, "-o", obj, *inc]
            if ptxas_verbose:
                cmd += ["-Xptxas", "-v"]
            jobs.append(cmd)
    for f in cpp:
        src = os.path.join(CSRC, f)
        obj = os.path.join(OBJ, f + ".o")
        objs.append(obj)
        if force or _stale(obj, [src] + hdr):
            jobs.append(["g++", "-O2", "-std=c++17", "-fPIC", "-Wall", *["-D" + d for d in defines], "-c", src, "-o", obj,
                         "-I", os.path.join(CUDA, "include"), *inc])
    if jobs:
        with cf.ThreadPoolExecutor(max_workers=os.cpu_count() or 4) as ex:
            res = list(ex.map(lambda c: subprocess.run(c, capture_output=True, text=True), jobs))
        for cmd, r in zip(jobs, res):
            if r.returncode != 0:
                sys.stderr.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
                raise RuntimeError(f"compile failed: {cmd[-1 - len(inc) - 2]}")
            if (not quiet or ptxas_verbose) and (r.stdout or r.stderr):
                sys.stderr.write(r.stdout + r.stderr)
    if force or jobs or _stale(SO, objs):
        lib = os.path.join(nccl, "lib")
        cmd = [NVCC, *ARCH, "-shared", "-o", SO, *objs, "-L", lib, "-l:libnccl.so.2",
               "-Xlinker", "-rpath=" + lib, "-cudart", "static"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
            raise RuntimeError("link failed")
    return SO


def build_devapi_test(force: bool = False) -> str:
    """tests/devapi/libxr_devapi_test.so: a TEST module that uses only the
    public device header include/xreduce_device.cuh."""
    src = os.path.join(ROOT, "tests", "devapi", "devapi_test.cu")
    so = os.path.join(ROOT, "tests", "devapi", "libxr_devapi_test.so")
    deps = [src] + [os.path.join(ROOT, "include", f) for f in os.listdir(os.path.join(ROOT, "include"))]
    if force or _stale(so, deps):
        cmd = [NVCC, *ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-shared",
               "--expt-relaxed-constexpr", src, "-o", so, "-cudart", "static"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
            raise RuntimeError("devapi test build failed")
    return so


if __name__ == "__main__":
    if "--variant" in sys.argv:  # A/B build: variants/libxreduce_<name>.so with -D defines
        i = sys.argv.index("--variant")
        name, defs = sys.argv[i + 1], [a[2:] for a in sys.argv[i + 2:] if a.startswith("-D")]
        vdir = os.path.join(ROOT, "variants")
        print(build(force=True, defines=defs, so_path=os.path.join(vdir, f"libxreduce_{name}.so"),
                    obj_dir=os.path.join(vdir, "obj_" + name)))
        sys.exit(0)
    print(build(force="--force" in sys.argv, ptxas_verbose="--ptxas-v" in sys.argv, quiet=False))
    print(build_devapi_test(force="--force" in sys.argv))
