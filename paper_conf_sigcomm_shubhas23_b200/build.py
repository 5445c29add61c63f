"""Build libadainf.so in-tree with nvcc for sm_100a only (no JIT, no other arch, no fast-math)."""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
# ADAINF_BUILD_OUT / ADAINF_BUILD_FLAGS: build a variant library elsewhere (A/B timing, -DADAINF_TIMING) without
# touching the in-tree one
OUT = os.environ.get("ADAINF_BUILD_OUT", os.path.join(HERE, "libadainf.so"))
BUILD = os.path.join(os.path.dirname(OUT), "_build") if "ADAINF_BUILD_OUT" in os.environ else os.path.join(HERE, "_build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _nccl_dir():
    try:
        import nvidia.nccl  # noqa: F401
        return os.path.dirname(nvidia.nccl.__file__) if nvidia.nccl.__file__ else list(nvidia.nccl.__path__)[0]
    except Exception:
        return None


FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
         "-Xcompiler", "-O2", "--expt-relaxed-constexpr", "-Xptxas", "-warn-spills",
         *os.environ.get("ADAINF_BUILD_FLAGS", "").split()]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _obj(src):
    return os.path.join(BUILD, os.path.basename(src)[:-3] + ".o")


def _deps_mtime():
    files = glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(
        os.path.join(HERE, "..", "include", "*.h"))
    return max(os.path.getmtime(f) for f in files)


def _compile(src, inc):
    obj = _obj(src)
    cmd = [NVCC, *FLAGS, *inc, "-c", src, "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
    return obj, r.stderr


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    nccl = _nccl_dir()
    inc = ["-I", CSRC, "-I", os.path.join(HERE, "..", "include")]
    if nccl:
        inc += ["-I", os.path.join(nccl, "include"), "-DADAINF_WITH_NCCL=1"]
    dm = _deps_mtime()
    todo = [s for s in sources() if force or not os.path.exists(_obj(s)) or os.path.getmtime(_obj(s)) < max(
        os.path.getmtime(s), dm)]
    if todo:
        with cf.ThreadPoolExecutor(max_workers=min(8, len(todo))) as ex:
            for obj, err in ex.map(lambda s: _compile(s, inc), todo):
                if verbose and err.strip():
                    print(err, file=sys.stderr)
    objs = [_obj(s) for s in sources()]
    if force or todo or not os.path.exists(OUT) or os.path.getmtime(OUT) < max(os.path.getmtime(o) for o in objs):
        link = [NVCC, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", OUT + ".tmp", *objs,
                "-lcudart"]
        if nccl:
            link += ["-L", os.path.join(nccl, "lib"), "-l:libnccl.so.2", "-Xlinker",
                     "-rpath=" + os.path.join(nccl, "lib")]
        r = subprocess.run(link, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("link failed:\n" + r.stderr)
        os.replace(OUT + ".tmp", OUT)
    return OUT


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
