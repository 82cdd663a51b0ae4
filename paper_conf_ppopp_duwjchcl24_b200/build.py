"""Build libliger.so in-tree: every CUDA/C++ source compiled for sm_100a with nvcc.

    python -m paper_conf_ppopp_duwjchcl24_b200.build
"""
import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
OBJ = os.path.join(HERE, "build")
LIB = os.path.join(HERE, "libliger.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
NCCL_INC = None
for cand in ("/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl/include", "/usr/include"):
    if os.path.exists(os.path.join(cand, "nccl.h")):
        NCCL_INC = cand
        break

FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall", "--expt-relaxed-constexpr"]


def _compile(src):
    obj = os.path.join(OBJ, os.path.basename(src) + ".o")
    deps = glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        [os.path.join(HERE, "..", "include", "liger.h")]
    if os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(p) for p in deps + [src]):
        return obj
    cmd = [NVCC, *FLAGS, "-c", src, "-o", obj]
    if NCCL_INC:
        cmd[1:1] = ["-I", NCCL_INC]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
    return obj


def build(verbose=False):
    os.makedirs(OBJ, exist_ok=True)
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))
    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        objs = list(ex.map(_compile, srcs))
    newest = max(os.path.getmtime(o) for o in objs)
    if not os.path.exists(LIB) or os.path.getmtime(LIB) < newest:
        cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", LIB + ".tmp", *objs, "-ldl",
               "-lpthread"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stderr}")
        os.replace(LIB + ".tmp", LIB)
    if verbose:
        print(LIB)
    return LIB


ORACLE_SRC = os.path.join(HERE, "..", "oracle", "layer_ref.cpp")


def build_oracle(out_dir=None, verbose=False):
    """Compile the fp32 C++ CPU oracle (oracle/layer_ref.cpp; test / baseline
    infrastructure, never loaded by the product): the timing binary `layer_ref` and
    the ctypes library `liblayer_ref.so` for its pin test.  -march=native: build it on
    the host that runs it (bench.py compiles its own copy on the GPU box's host)."""
    out_dir = out_dir or os.path.join(HERE, "..", "oracle")
    os.makedirs(out_dir, exist_ok=True)
    exe = os.path.join(out_dir, "layer_ref")
    so = os.path.join(out_dir, "liblayer_ref.so")
    base = ["g++", "-O3", "-march=native", "-fopenmp", "-std=c++17", ORACLE_SRC]
    for cmd, out in ((base + ["-o", exe], exe), (base + ["-DLAYER_REF_NO_MAIN", "-shared", "-fPIC", "-o", so], so)):
        if os.path.exists(out) and os.path.getmtime(out) >= os.path.getmtime(ORACLE_SRC):
            continue
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"g++ failed for the CPU oracle:\n{r.stderr}")
    if verbose:
        print(exe)
    return exe, so


if __name__ == "__main__":
    build(verbose=True)
    build_oracle(verbose=True)
    sys.exit(0)
