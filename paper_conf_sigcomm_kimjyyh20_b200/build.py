"""Build libsr.so (all CUDA sources, sm_100a) in-tree: `python -m paper_conf_sigcomm_kimjyyh20_b200.build`."""
import os
import shutil
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libsr.so")
SOURCES = ["conv.cu", "conv_roll.cu", "conv_block.cu", "conv_block2.cu", "conv_block_split.cu", "conv_bodytail.cu", "conv_wgrad.cu", "kernels.cu", "sr.cu", "test_kernels.cu"]
OBJDIR = os.path.join(ROOT, "build", "obj")


def nvcc_path():
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def needs_rebuild():
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(ROOT, "include", "sr.h")]
    return any(os.path.getmtime(d) > t for d in deps if os.path.exists(d))


def build(force=False, verbose=True):
    """Compile every translation unit to an object in parallel (build/obj), then link libsr.so."""
    if not force and not needs_rebuild():
        return LIB
    os.makedirs(OBJDIR, exist_ok=True)
    flags = ["-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-Xcompiler", "-fPIC",
             "-Xptxas", "-v" if os.environ.get("SR_PTXAS_V") else "-O3", "-I", os.path.join(ROOT, "include")]
    flags += os.environ.get("SR_NVCC_DEFS", "").split()  # A/B builds only, e.g. "-DSR_BLOCK_DIRECT_OUT=1"
    nvcc = nvcc_path()

    def compile_one(src):
        obj = os.path.join(OBJDIR, src.replace(".cu", ".o"))
        cmd = [nvcc] + flags + ["-c", os.path.join(CSRC, src), "-o", obj]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        r = subprocess.run(cmd, cwd=CSRC, capture_output=True, text=True)
        if r.stderr:
            print(r.stderr, file=sys.stderr, end="")
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed on {src}")
        return obj

    with ThreadPoolExecutor(max_workers=min(len(SOURCES), os.cpu_count() or 4)) as ex:
        objs = list(ex.map(compile_one, SOURCES))
    cmd = [nvcc, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", LIB + ".tmp"] + objs
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.run(cmd, check=True, cwd=CSRC)
    os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv)
