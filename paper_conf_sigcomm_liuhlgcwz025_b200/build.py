"""Build the ResCCL native library in-tree.

  libresccl.so     C++ planner + codegen + control plane + C ABI (g++), linked against
                   static cudart and NVRTC; the generated kernels are compiled by NVRTC
                   for sm_100a at load time.
  build/selftest_ring_ar2.cubin
                   nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo compile of a
                   generated ring AllReduce kernel (the "does the CUDA build" check that
                   runs without a GPU).

Usage: python -m paper_conf_sigcomm_liuhlgcwz025_b200.build [--force]
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
BUILD = os.path.join(HERE, "build")
LIB = os.path.join(HERE, "libresccl.so")
SHIM = os.path.join(HERE, "libresccl_nccl.so")   # NCCL-symbol shim (include/resccl_nccl.h)
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")

SOURCES = [
    "plan/ir.cc",
    "plan/plan.cc",
    "plan/codegen.cc",
    "plan/rescclang.cc",
    "plan/timeline.cc",
    "comm/comm.cc",
]
HEADERS = [
    "plan/ir.h", "plan/plan.h", "plan/codegen.h", "plan/timeline.h", "device/resccl_device.cuh",
]


def _run(cmd):
    r = subprocess.run(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
    if r.returncode != 0:
        raise RuntimeError("command failed: " + " ".join(cmd) + "\n" + r.stdout)
    return r.stdout


def _embed_device_src():
    src = open(os.path.join(CSRC, "device", "resccl_device.cuh")).read()
    delim = "RESCCL_DEVSRC"
    assert ")" + delim not in src
    out = os.path.join(CSRC, "comm", "device_src.inc")
    body = 'R"' + delim + "(" + src + ")" + delim + '"\n'
    if not os.path.exists(out) or open(out).read() != body:
        with open(out, "w") as f:
            f.write(body)
    return out


def _newer(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    inc = _embed_device_src()
    hdrs = [os.path.join(CSRC, h) for h in HEADERS] + [inc, os.path.join(ROOT, "include", "resccl.h")]
    objs = []
    for s in SOURCES:
        src = os.path.join(CSRC, s)
        obj = os.path.join(BUILD, s.replace("/", "_").replace(".cc", ".o"))
        objs.append(obj)
        if force or _newer(obj, [src] + hdrs):
            cmd = ["g++", "-O2", "-g", "-std=c++17", "-fPIC", "-Wall", "-Wno-unused-function",
                   "-I", os.path.join(CUDA, "include"), "-c", src, "-o", obj]
            if verbose:
                print(" ".join(cmd))
            _run(cmd)
    if force or _newer(LIB, objs):
        cmd = ["g++", "-shared", "-o", LIB] + objs + [
            "-L", os.path.join(CUDA, "lib64"), "-lcudart_static", "-lnvrtc", "-ldl", "-lrt", "-lpthread",
            "-Wl,-rpath," + os.path.join(CUDA, "lib64"), "-Wl,--no-undefined"]
        if verbose:
            print(" ".join(cmd))
        _run(cmd)
    shim_src = os.path.join(CSRC, "shim", "nccl_shim.cc")
    shim_hdrs = [os.path.join(ROOT, "include", "resccl_nccl.h"), os.path.join(ROOT, "include", "resccl.h")]
    if force or _newer(SHIM, [shim_src, LIB] + shim_hdrs):
        cmd = ["g++", "-O2", "-g", "-std=c++17", "-fPIC", "-Wall", "-shared", "-I", os.path.join(ROOT, "include"),
               shim_src, "-o", SHIM, "-L", HERE, "-lresccl", "-ldl", "-lpthread", "-Wl,-rpath,$ORIGIN",
               "-Wl,--no-undefined"]
        if verbose:
            print(" ".join(cmd))
        _run(cmd)
    return LIB


def selftest_cubin() -> str:
    """Generate a ring AllReduce (N=2) kernel with the library and compile it with nvcc
    for sm_100a -- proves the device library + generator output build offline."""
    lib = ctypes.CDLL(LIB)
    lib.rescclGenerateIr.restype = ctypes.c_int
    lib.rescclCodegenIr.restype = ctypes.c_int
    n = ctypes.c_size_t(1 << 20)
    ir = ctypes.create_string_buffer(n.value)
    if lib.rescclGenerateIr(b"ring", 2, 2, None, ir, ctypes.byref(n)) != 0:
        raise RuntimeError("rescclGenerateIr failed")
    n = ctypes.c_size_t(1 << 24)
    src = ctypes.create_string_buffer(n.value)
    if lib.rescclCodegenIr(ir.value, b"chunkbytes=4096 instances=2", 0, 2, src, ctypes.byref(n)) != 0:
        raise RuntimeError("rescclCodegenIr failed")
    cu = os.path.join(BUILD, "selftest_ring_ar2.cu")
    with open(cu, "w") as f:
        f.write(src.value.decode())
    cubin = os.path.join(BUILD, "selftest_ring_ar2.cubin")
    _run([NVCC, "-cubin", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
          "-I", os.path.join(CSRC, "device"), "-DRESCCL_T=rdev::TBF16", "-DRESCCL_OP=0", "-Xptxas", "-v",
          cu, "-o", cubin])
    # f3: the NVLS kernel (multimem.ld_reduce / multimem.st), bf16 sum AllReduce
    nv = os.path.join(BUILD, "selftest_nvls_ar.cu")
    with open(nv, "w") as f:
        f.write('#include "resccl_device.cuh"\n'
                'extern "C" __global__ void __launch_bounds__(512, 1) resccl_nvls_kernel(rdev::NvlsArgs a) {\n'
                '  rdev::nvls_run<RESCCL_T, RESCCL_OP, 2>(a);\n}\n')
    _run([NVCC, "-cubin", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
          "-I", os.path.join(CSRC, "device"), "-DRESCCL_T=rdev::TBF16", "-DRESCCL_OP=0", "-Xptxas", "-v",
          nv, "-o", os.path.join(BUILD, "selftest_nvls_ar.cubin")])
    return cubin


if __name__ == "__main__":
    p = build(force="--force" in sys.argv, verbose=True)
    print("built", p)
    print("selftest", selftest_cubin())
