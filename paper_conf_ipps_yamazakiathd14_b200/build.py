"""Build libcagmres.so in-tree: nvcc for sm_100a (B200) + the host C++ sources.

    python -m paper_conf_ipps_yamazakiathd14_b200.build

The library links NCCL from the nvidia-nccl wheel torch itself loads (same soname), with an
rpath so it also loads without torch.  Oracle code is never compiled into it.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libcagmres.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_dirs():
    cands = []
    try:
        import nvidia.nccl as nn  # type: ignore
        base = list(nn.__path__)[0]
        cands.append((os.path.join(base, "include"), os.path.join(base, "lib")))
    except Exception:
        pass
    cands.append(("/usr/include", "/usr/lib/x86_64-linux-gnu"))
    for inc, lib in cands:
        if os.path.exists(os.path.join(inc, "nccl.h")) and glob.glob(os.path.join(lib, "libnccl.so*")):
            return inc, lib
    raise RuntimeError("nccl.h / libnccl.so not found")


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.h")) + [os.path.join(ROOT, "include", "cagmres.h")]
    return any(os.path.getmtime(p) > t for p in deps)


def build(verbose: bool = False, force: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    inc, lib = _nccl_dirs()
    nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
    libdir = lib
    nccl_so = sorted(glob.glob(os.path.join(lib, "libnccl.so*")))
    link = ["-L", libdir, "-l:" + os.path.basename(nccl_so[0])] if not os.path.exists(
        os.path.join(libdir, "libnccl.so")) else ["-L", libdir, "-lnccl"]
    common = ["-O3", *ARCH, "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3",
              "-Xptxas", "-v" if verbose else "-O3", "-I", os.path.join(ROOT, "include"), "-I", inc]
    objdir = os.path.join(ROOT, "build", "obj")
    os.makedirs(objdir, exist_ok=True)

    def compile_one(src):
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        r = subprocess.run([nvcc, *common, "-c", src, "-o", obj], capture_output=True, text=True)
        return src, obj, r

    # one nvcc per translation unit, in parallel (no cross-TU device code: no -rdc needed)
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=min(16, os.cpu_count() or 4)) as ex:
        results = list(ex.map(compile_one, sources()))
    for src, _, r in results:
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError(f"nvcc build of {os.path.basename(src)} failed")
        if verbose:
            sys.stderr.write(r.stderr)
    cmd = [nvcc, *ARCH, "-shared", "-Xcompiler", "-fPIC", *[o for _, o, _ in results], *link,
           "-Xlinker", "-rpath," + libdir, "-lcudart", "-o", LIB + ".tmp"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("link of libcagmres.so failed")
    os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    build(verbose="-v" in sys.argv, force=True)
    print(LIB)
