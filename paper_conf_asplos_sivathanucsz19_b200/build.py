"""Build the in-tree C-ABI library `lib/libastra.so` for sm_100a (nvcc, no JIT cache).

Every .cu/.cpp under csrc/ is compiled with
    nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3
and linked against the CUDA runtime and the NCCL shipped with the venv (rpath set), so the
library travels to the GPU box with the repository snapshot.
"""
from __future__ import annotations

import glob
import hashlib
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
OUT_DIR = os.path.join(HERE, "lib")
OUT = os.path.join(OUT_DIR, "libastra.so")
BUILD = os.path.join(HERE, "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_dir():
    import nvidia.nccl as n  # shipped with torch
    return os.path.dirname(n.__file__) if getattr(n, "__file__", None) else list(n.__path__)[0]


def sources():
    s = sorted(glob.glob(os.path.join(CSRC, "**", "*.cu"), recursive=True))
    s += sorted(glob.glob(os.path.join(CSRC, "**", "*.cpp"), recursive=True))
    return s


def headers():
    h = glob.glob(os.path.join(CSRC, "**", "*.h"), recursive=True)
    h += glob.glob(os.path.join(CSRC, "**", "*.cuh"), recursive=True)
    h += glob.glob(os.path.join(ROOT, "include", "*.h"))
    return sorted(h)


def _digest(paths, extra=""):
    m = hashlib.sha256(extra.encode())
    for p in paths:
        with open(p, "rb") as f:
            m.update(p.encode())
            m.update(f.read())
    return m.hexdigest()


def build(verbose=False, force=False):
    nd = nccl_dir()
    inc = ["-I", os.path.join(ROOT, "include"), "-I", os.path.join(nd, "include")]
    flags = ["-std=c++17", "-O3", "-lineinfo", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr"] + ARCH + inc
    os.makedirs(BUILD, exist_ok=True)
    os.makedirs(OUT_DIR, exist_ok=True)
    hdr_digest = _digest(headers(), " ".join(flags))
    objs = []
    jobs = []
    for src in sources():
        rel = os.path.relpath(src, CSRC).replace(os.sep, "_")
        obj = os.path.join(BUILD, rel + ".o")
        stamp = obj + ".sha"
        dig = _digest([src], hdr_digest)
        objs.append(obj)
        if not force and os.path.exists(obj) and os.path.exists(stamp) and open(stamp).read() == dig:
            continue
        cmd = [NVCC] + flags + ["-c", src, "-o", obj]
        if src.endswith(".cpp"):
            cmd = [NVCC, "-x", "cu"] + flags + ["-c", src, "-o", obj]
        jobs.append((cmd, stamp, dig, src))

    def run(job):
        cmd, stamp, dig, src = job
        if verbose:
            print(" ".join(cmd), flush=True)
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
        with open(stamp, "w") as f:
            f.write(dig)
        return src

    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 2)) as ex:
        for s in ex.map(run, jobs):
            if verbose:
                print("built", os.path.relpath(s, HERE), flush=True)
    libdir = os.path.join(nd, "lib")
    link = [NVCC] + ARCH + ["-shared", "-o", OUT] + objs + [
        "-L", libdir, "-l:libnccl.so.2", "-Xlinker", "-rpath=" + libdir, "-lcudart"]
    if jobs or not os.path.exists(OUT):
        r = subprocess.run(link, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("link failed:\n" + r.stdout + r.stderr)
    return OUT


if __name__ == "__main__":
    print(build(verbose="-v" in sys.argv, force="-f" in sys.argv))
