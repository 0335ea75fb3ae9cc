"""Build libfop.so in-tree (host C++ planner/codegen/runtime + the embedded
sm_100a device header), and check every kernel skeleton with nvcc for
sm_100a.

    python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build

The kernels themselves are generated per fused operator at fop_plan time and
compiled with NVRTC for sm_100a (-arch=sm_100a -lineinfo); ``nvcc_check``
compiles the generated sources of the five configs with nvcc
(-gencode arch=compute_100a,code=sm_100a -lineinfo) as an independent check
and leaves the cubins under build/kernels/ for cuobjdump.
"""
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libfop.so")
BUILD = os.path.join(ROOT, "build")


def _embed_header():
    src = os.path.join(CSRC, "device", "fop_device.cuh")
    text = open(src).read()
    assert ')FOPDEV"' not in text
    os.makedirs(BUILD, exist_ok=True)
    out = os.path.join(BUILD, "fop_device_embed.cpp")
    body = ('// generated from csrc/device/fop_device.cuh by build.py\n'
            'namespace fop { extern const char* kDeviceHeader; '
            'const char* kDeviceHeader = R"FOPDEV(' + text + ')FOPDEV"; }\n')
    if not os.path.exists(out) or open(out).read() != body:
        with open(out, "w") as f:
            f.write(body)
    return out


def build(force=False, verbose=False):
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cpp")))
    deps = srcs + glob.glob(os.path.join(CSRC, "*.h")) + \
        glob.glob(os.path.join(CSRC, "device", "*.cuh")) + [os.path.join(ROOT, "include", "fop.h")]
    emb = _embed_header()
    if not force and os.path.exists(LIB):
        t = os.path.getmtime(LIB)
        if all(os.path.getmtime(p) <= t for p in deps):
            return LIB
    cmd = ["g++", "-O2", "-g", "-std=c++17", "-fPIC", "-shared", "-Wall", "-Wno-unused-function",
           "-fvisibility=hidden", "-I", os.path.join(ROOT, "include")] + srcs + [emb] + \
        ["-o", LIB + ".tmp", "-ldl", "-lpthread"]
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(LIB + ".tmp", LIB)
    return LIB


def nvcc_check(sources, out_dir=None):
    """Compile generated kernel sources with nvcc for sm_100a (cubin)."""
    out_dir = out_dir or os.path.join(BUILD, "kernels")
    os.makedirs(out_dir, exist_ok=True)
    inc = os.path.join(CSRC, "device")
    cubins = []
    for name, src in sources:
        cu = os.path.join(out_dir, name + ".cu")
        with open(cu, "w") as f:
            f.write(src)
        cub = os.path.join(out_dir, name + ".cubin")
        subprocess.check_call(["nvcc", "-cubin", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a",
                               "-lineinfo", "-O3", "-fmad=false", "-I", inc, "-o", cub, cu])
        cubins.append(cub)
    return cubins


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
