"""Build libsnicit.so for sm_100a with nvcc (in-tree, so the .so travels with the repo)."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
OUT = os.path.join(HERE, "lib", "libsnicit.so")
SOURCES = ["snicit_api.cu", "kernels_layer.cu", "kernels_gen.cu", "kernels_pre_fused.cu", "kernels_pre_pair.cu", "kernels_pre_cluster.cu", "kernels_const.cu", "kernels_circ.cu", "kernels_circ_seg.cu", "kernels_circ_col.cu", "kernels_post.cu", "kernels_convert.cu"]
HEADERS = ["snicit_internal.cuh", os.path.join("..", "..", "include", "snicit.h")]
NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
              "-Xcompiler", "-fPIC", "-shared"]


def nvcc_path() -> str:
    for p in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc"):
        if p and os.path.exists(p):
            return p
    return "nvcc"


def build(force: bool = False, verbose: bool = False) -> str:
    """Compile each .cu to an object in parallel (only those older than their sources/headers unless
    `force`), then link libsnicit.so."""
    from concurrent.futures import ThreadPoolExecutor

    hdr_t = max(os.path.getmtime(os.path.join(CSRC, h)) for h in HEADERS)
    objdir = os.path.join(HERE, "lib", "obj")
    os.makedirs(objdir, exist_ok=True)
    objs = [os.path.join(objdir, s[:-3] + ".o") for s in SOURCES]
    stale = [i for i, (s, o) in enumerate(zip(SOURCES, objs))
             if force or not os.path.exists(o) or os.path.getmtime(o) < max(hdr_t, os.path.getmtime(os.path.join(CSRC, s)))]
    if not stale and os.path.exists(OUT) and os.path.getmtime(OUT) >= max(os.path.getmtime(o) for o in objs):
        return OUT
    flags = [f for f in NVCC_FLAGS if f != "-shared"]

    def compile_one(i: int) -> None:
        cmd = [nvcc_path()] + flags + (["-Xptxas", "-v"] if verbose else []) + ["-c", SOURCES[i], "-o", objs[i] + ".tmp"]
        subprocess.check_call(cmd, cwd=CSRC)
        os.replace(objs[i] + ".tmp", objs[i])

    with ThreadPoolExecutor(max_workers=max(1, min(len(stale), os.cpu_count() or 1))) as ex:
        list(ex.map(compile_one, stale))
    tmp = OUT + ".tmp"
    subprocess.check_call([nvcc_path(), "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp] + objs, cwd=CSRC)
    os.replace(tmp, OUT)
    return OUT


if __name__ == "__main__":
    import sys
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
