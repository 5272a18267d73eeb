"""Build libalgas.so in-tree with nvcc for sm_100a (no JIT cache: the .so
travels with the repo snapshot to the GPU box)."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
# ALGAS_LIB: load / build an alternative library file (A/B builds of the
# same sources with extra -D flags from ALGAS_BUILD_DEFS, e.g. build/*.so)
LIB = os.environ.get("ALGAS_LIB") or os.path.join(HERE, "libalgas.so")
EXTRA_DEFS = os.environ.get("ALGAS_BUILD_DEFS", "").split()
SOURCES = ["search_kernels.cu", "search_api.cu", "runtime.cu", "knn.cu", "build_part.cu", "knn_tc.cu"]
# the search kernels, one object per thread count (compiled in parallel)
THREAD_COUNTS = [32, 64, 128, 256, 512, 1024]
KERNEL_TU = "kernels_nt.cu"
HEADERS = ["search_core.cuh", "kernels.cuh", "internal.h", KERNEL_TU, os.path.join("..", "..", "include", "algas.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
         "--expt-relaxed-constexpr", "-Xptxas", "-v"]


def source_hash() -> str:
    """sha256 over the library's sources, headers, kernel unit and this file
    (content, not mtimes: a repo snapshot copied to another machine keeps
    its hash but not necessarily its mtimes)."""
    import hashlib
    h = hashlib.sha256()
    for f in SOURCES + HEADERS + ["../build.py"]:
        with open(os.path.join(CSRC, f), "rb") as fh:
            h.update(f.encode() + b"\0" + fh.read())
    h.update(" ".join(EXTRA_DEFS).encode())
    return h.hexdigest()


def _hash_path() -> str:
    return LIB + ".srchash"


def built_hash() -> str | None:
    try:
        with open(_hash_path()) as f:
            return f.read().strip()
    except OSError:
        return None


def _stale() -> bool:
    return not os.path.exists(LIB) or built_hash() != source_hash()


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    objs = []
    jobs = []
    tag = f".{os.getpid()}" if EXTRA_DEFS else ""
    units = [(src, src.replace(".cu", f"{tag}.o"), []) for src in SOURCES]
    units += [(KERNEL_TU, f"kernels_nt{nt}{tag}.o", [f"-DALGAS_NT={nt}"]) for nt in THREAD_COUNTS]
    for src, o, defs in units:
        obj = os.path.join(CSRC, o)
        cmd = [NVCC, *ARCH, *FLAGS, *EXTRA_DEFS, *defs, "-c", os.path.join(CSRC, src), "-o", obj]
        jobs.append((f"{src} {' '.join(defs)}", subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)))
        objs.append(obj)
    logs = []
    failed = False
    for src, p in jobs:
        out, _ = p.communicate()
        logs.append(f"== {src}\n{out}")
        if p.returncode != 0:
            failed = True
    log_path = LIB[:-3] + ".build.log" if EXTRA_DEFS else os.path.join(HERE, "build.log")
    with open(log_path, "w") as f:
        f.write("\n".join(logs))
    if failed:
        sys.stderr.write("\n".join(logs)[-20000:])
        raise RuntimeError(f"nvcc failed (see {log_path})")
    tmp = LIB + f".tmp{os.getpid()}"
    # cuBLAS (tensor-core kNN screen) from the toolkit; rpath so the library
    # resolves it without LD_LIBRARY_PATH (same image on the GPU box)
    cuda_lib = os.path.join(os.path.dirname(os.path.dirname(NVCC)), "lib64")
    subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart_static", "-L" + cuda_lib, "-lcublas",
                           "-Xlinker", "-rpath=" + cuda_lib, "-lrt", "-lpthread", "-ldl"])
    os.replace(tmp, LIB)
    with open(_hash_path(), "w") as f:
        f.write(source_hash() + "\n")
    for o in objs:
        os.remove(o)
    if verbose:
        print("\n".join(logs))
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
