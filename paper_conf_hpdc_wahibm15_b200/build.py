"""In-tree build of libstencilfuse.so (host C++ + NVRTC JIT of sm_100a kernels).

  python -m paper_conf_hpdc_wahibm15_b200.build      (or __graft_entry__.build())

Steps: embed csrc/device/sf_device.cuh as a string (NVRTC header of every
generated kernel); nvcc-compile that header once AOT for sm_100a as a
self-check (and keep its SASS under build/ for inspection); compile the host
sources; link against the static CUDA runtime, NVRTC and NCCL (rpath), so the
library loads on GPU-less hosts and binds the driver lazily.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
BUILD = os.path.join(HERE, "build")
LIB = os.path.join(HERE, "libstencilfuse.so")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")


def nccl_dir():
    try:
        import nvidia.nccl as m
        return os.path.dirname(m.__file__) if m.__file__ else list(m.__path__)[0]
    except Exception:
        d = os.path.join(sys.prefix, "lib", f"python{sys.version_info.major}.{sys.version_info.minor}",
                         "site-packages", "nvidia", "nccl")
        return d


def _run(cmd):
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"build failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    return r


def embed_header():
    """csrc/sf_device_embed.inc: the device header as a C++ raw string (the NVRTC header of
    every generated kernel).  Generated here at every build, never edited or tracked."""
    src = open(os.path.join(CSRC, "device", "sf_device.cuh")).read()
    out = os.path.join(CSRC, "sf_device_embed.inc")
    text = 'R"SFDEV(' + src + ')SFDEV"\n'
    if not os.path.exists(out) or open(out).read() != text:
        open(out, "w").write(text)


def device_selfcheck():
    """nvcc -gencode arch=compute_100a,code=sm_100a on the device primitives."""
    os.makedirs(BUILD, exist_ok=True)
    src = os.path.join(CSRC, "device", "sf_device_check.cu")
    cub = os.path.join(BUILD, "sf_device_check.cubin")
    if os.path.exists(cub) and os.path.getmtime(cub) >= max(
            os.path.getmtime(src), os.path.getmtime(os.path.join(CSRC, "device", "sf_device.cuh"))):
        return cub
    _run([os.path.join(CUDA, "bin", "nvcc"), "-gencode", "arch=compute_100a,code=sm_100a",
          "-lineinfo", "-O3", "-cubin", "-Xptxas", "-v", "-I", os.path.join(CSRC, "device"),
          "-o", cub, src])
    return cub


def build(force: bool = False, verbose: bool = False) -> str:
    embed_header()
    device_selfcheck()
    os.makedirs(BUILD, exist_ok=True)
    nd = nccl_dir()
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cpp")))
    deps = srcs + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.inc")) + \
        [os.path.join(ROOT, "include", "stencilfuse.h")]
    if not force and os.path.exists(LIB) and \
            os.path.getmtime(LIB) >= max(os.path.getmtime(d) for d in deps):
        return LIB
    cflags = ["-O2", "-g", "-std=c++17", "-fPIC", "-Wall", "-Wno-unused-function",
              "-I", os.path.join(ROOT, "include"), "-I", CSRC,
              "-I", os.path.join(CUDA, "include"), "-I", os.path.join(nd, "include")]
    objs = []

    def cc(src):
        obj = os.path.join(BUILD, os.path.basename(src)[:-4] + ".o")
        _run(["g++"] + cflags + ["-c", src, "-o", obj])
        return obj

    with cf.ThreadPoolExecutor(max_workers=os.cpu_count() or 4) as ex:
        objs = list(ex.map(cc, srcs))
    _run(["g++", "-shared", "-o", LIB] + objs + [
        os.path.join(CUDA, "lib64", "libcudart_static.a"),
        "-L", os.path.join(CUDA, "lib64"), "-lnvrtc",
        "-L", os.path.join(nd, "lib"), "-l:libnccl.so.2",
        f"-Wl,-rpath,{os.path.join(CUDA, 'lib64')}", f"-Wl,-rpath,{os.path.join(nd, 'lib')}",
        "-ldl", "-lpthread", "-lrt"])
    if verbose:
        print("built", LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
