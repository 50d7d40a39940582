"""Build libopp.so in-tree with nvcc for sm_100a (no JIT, no torch extension).

python -m paper_conf_icpp_lantra0m24_b200.build   (also called by
__graft_entry__.build()).
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.environ.get("OPP_LIB_OUT", os.path.join(HERE, "libopp.so"))
SOURCES = ["opp.cu", "opp_kernels.cu", "opp_comm.cu", "opp_field.cu", "opp_em.cu", "opp_boltz.cu"]
HEADERS = ["opp_internal.h", "opp_kernels.h", "opp_comm.h", "opp_field.h", "opp_em.h"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _nccl_dir():
    """torch's pip NCCL (2.28.x): the one NCCL loaded in a torch process."""
    try:
        import importlib.util
        spec = importlib.util.find_spec("nvidia.nccl")
        if spec and spec.submodule_search_locations:
            d = list(spec.submodule_search_locations)[0]
            if os.path.exists(os.path.join(d, "include", "nccl.h")):
                return d
    except Exception:   # noqa: BLE001
        pass
    return None
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2,-Wall",
         "--expt-relaxed-constexpr", "-Xptxas", "-v", "-I", os.path.join(ROOT, "include"),
         "-I", CSRC] + os.environ.get("OPP_NVCC_EXTRA", "").split()


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "opp.h")]
    return any(os.path.getmtime(d) > t for d in deps if os.path.exists(d))


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    objs = []
    # objects of an alternative build (OPP_LIB_OUT) live apart from the in-tree library's
    odir = os.path.join(ROOT, "build") if "OPP_LIB_OUT" not in os.environ else \
        os.path.join(ROOT, "build", os.path.splitext(os.path.basename(LIB))[0])
    os.makedirs(odir, exist_ok=True)
    nccl = _nccl_dir()
    extra, link = [], []
    if nccl:
        extra = ["-DOPP_WITH_NCCL", "-I", os.path.join(nccl, "include")]
        link = ["-L", os.path.join(nccl, "lib"), "-l:libnccl.so.2",
                "-Xlinker", "-rpath=" + os.path.join(nccl, "lib")]
    for src in SOURCES:
        obj = os.path.join(odir, src.replace(".cu", ".o"))
        cmd = [NVCC, *ARCH, *FLAGS, *extra, "-c", os.path.join(CSRC, src), "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError(f"nvcc failed on {src}")
        if verbose:
            sys.stderr.write(r.stderr)
        objs.append(obj)
    cmd = [NVCC, *ARCH, "-shared", "-o", LIB, *objs, "-cudart", "static", *link]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("link failed")
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
