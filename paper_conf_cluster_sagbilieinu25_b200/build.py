"""Build libuniconn_b200.so in-tree with nvcc for sm_100a (no torch extension machinery).

    python paper_conf_cluster_sagbilieinu25_b200/build.py [--force] [--define X=Y --out path.so]

(run it as a script, not with -m: importing the package loads the library being built)

The library links the NCCL shipped in the torch wheel (``nvidia/nccl``, 2.28.x) with an rpath
to it, and CUDA's static runtime (nvcc default), so it loads beside torch in one process.
"""
from __future__ import annotations

import glob
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libuniconn_b200.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall",
              "-Xptxas", "-v", "--expt-relaxed-constexpr"]


def nccl_dir() -> str:
    import importlib.util
    spec = importlib.util.find_spec("nvidia.nccl")
    if spec is None or not spec.submodule_search_locations:
        raise RuntimeError("nvidia.nccl (torch's NCCL wheel) not found")
    return list(spec.submodule_search_locations)[0]


def nvcc() -> str:
    for cand in (shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found")


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        [os.path.join(INCLUDE, "uniconn.h"), __file__]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """Build the library.  `defines` (e.g. ["UC_KR=8"]) and `out` produce A/B builds of the same
    sources (compile-time tuning knobs in csrc/kernels.cu), loaded with UC_LIB_PATH=<out>."""
    target = out or LIB
    if not force and not defines and out is None and not _stale():
        if any(not os.path.exists(t) or os.path.getmtime(t) < os.path.getmtime(s) for s, t in _example_targets()):
            build_examples()
        build_native()
        return LIB
    nd = nccl_dir()
    os.makedirs(os.path.dirname(os.path.abspath(target)), exist_ok=True)
    tmp = target + f".tmp{os.getpid()}"
    objdir = os.path.join(ROOT, "build", "obj", os.path.basename(target) + f".{os.getpid()}")
    os.makedirs(objdir, exist_ok=True)
    flags = [*ARCH, *NVCC_FLAGS, *[f"-D{d}" for d in defines], "-I", INCLUDE, "-I", CSRC,
             "-I", os.path.join(nd, "include")]
    # one nvcc per translation unit, in parallel (the kernel TUs dominate the build time)
    jobs = [(src, os.path.join(objdir, os.path.basename(src) + ".o")) for src in sources()]
    cmds = [[nvcc(), *flags, "-c", src, "-o", obj] for src, obj in jobs]
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=max(1, min(len(cmds), os.cpu_count() or 1))) as ex:
        results = list(ex.map(lambda c: subprocess.run(c, capture_output=True, text=True), cmds))
    link = [nvcc(), *ARCH, "-shared", *[o for _, o in jobs], "-o", tmp, "-L", os.path.join(nd, "lib"),
            "-l:libnccl.so.2", "-Xlinker", "-rpath=" + os.path.join(nd, "lib")]
    if all(r.returncode == 0 for r in results):
        results.append(subprocess.run(link, capture_output=True, text=True))
        cmds.append(link)
    log = os.path.join(CSRC, "build.log")
    with open(log, "w") as f:
        for c, r in zip(cmds, results):
            f.write(" ".join(c) + "\n" + r.stdout + r.stderr)
    shutil.rmtree(objdir, ignore_errors=True)
    if any(r.returncode != 0 for r in results):
        sys.stderr.write("".join(r.stdout + r.stderr for r in results if r.returncode != 0))
        raise RuntimeError(f"nvcc failed (see {log})")
    if verbose:
        sys.stderr.write("".join(r.stderr for r in results))
    os.replace(tmp, target)
    if out is None:
        build_examples()
        build_native()
    return target


def _example_targets():
    ex = os.path.join(ROOT, "examples")
    t = [(s, s[:-2]) for s in glob.glob(os.path.join(ex, "*.c"))]
    t += [(s, os.path.join(ex, "lib" + os.path.basename(s)[:-3].replace("device_api_ring", "uc_device_example") + ".so"))
          for s in glob.glob(os.path.join(ex, "*.cu"))]
    return t


NATIVE = os.path.join(ROOT, "benchmarks", "native")


def build_native(force: bool = False) -> str:
    """In-box comparator (not the product): the Listing-3 Jacobi on NCCL's device
    API, benchmarks/native/nccl_dev_jacobi.cu -> libuc_nccl_dev.so (nvcc sm_100a, the wheel's NCCL)."""
    src = os.path.join(NATIVE, "nccl_dev_jacobi.cu")
    out = os.path.join(NATIVE, "libuc_nccl_dev.so")
    deps = [src, os.path.join(NATIVE, "nccl_dev_jacobi.h"), __file__]
    if not force and os.path.exists(out) and all(os.path.getmtime(d) <= os.path.getmtime(out) for d in deps):
        return out
    nd = nccl_dir()
    subprocess.check_call([nvcc(), *ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-shared",
                           "-I", os.path.join(nd, "include"), src, "-o", out, "-L", os.path.join(nd, "lib"),
                           "-l:libnccl.so.2", "-Xlinker", "-rpath=" + os.path.join(nd, "lib")])
    return out


def build_examples() -> None:
    """Users of the library: plain-C drivers of the C-ABI (examples/*.c, gcc) and user kernels
    written against the header-only device API (examples/*.cu, nvcc sm_100a, shared library)."""
    for src, target in _example_targets():
        if src.endswith(".c"):
            subprocess.check_call(["gcc", "-O2", "-std=c11", "-I", INCLUDE, src, "-o", target, "-L", PKG,
                                   "-l:libuniconn_b200.so", "-Wl,-rpath," + PKG])
        else:
            subprocess.check_call([nvcc(), *ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-shared",
                                   "-I", INCLUDE, src, "-o", target])


if __name__ == "__main__":
    import argparse
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-v", action="store_true")
    ap.add_argument("--define", action="append", default=[])
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    print(build(force=a.force, verbose=a.v, defines=a.define, out=a.out))
