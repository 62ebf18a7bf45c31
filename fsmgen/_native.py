"""Build + load the generator's native helpers (host C and device CUDA).

Workload generation only; see fsmgen/csrc/*.  Both libraries are built in-tree so that they
travel to the GPU box with the repo snapshot.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

_HERE = os.path.dirname(os.path.abspath(__file__))
HOST_SO = os.path.join(_HERE, "libfsmgen.so")
DEV_SO = os.path.join(_HERE, "libfsmgen_dev.so")
_HOST_SRC = os.path.join(_HERE, "csrc", "fsmgen.c")
_DEV_SRC = os.path.join(_HERE, "csrc", "fsmgen_dev.cu")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _stale(so: str, src: str) -> bool:
    return not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src)


def build_host(force: bool = False) -> str:
    if force or _stale(HOST_SO, _HOST_SRC):
        subprocess.check_call(["gcc", "-O3", "-shared", "-fPIC", "-o", HOST_SO, _HOST_SRC])
    return HOST_SO


def build_dev(force: bool = False) -> str:
    if force or _stale(DEV_SO, _DEV_SRC):
        subprocess.check_call([
            NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo",
            "-shared", "-Xcompiler", "-fPIC", "-o", DEV_SO, _DEV_SRC])
    return DEV_SO


_host = None
_dev = None


def host_lib() -> ctypes.CDLL:
    global _host
    if _host is None:
        lib = ctypes.CDLL(build_host())
        lib.fsmgen_word.restype = ctypes.c_uint64
        lib.fsmgen_word.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        lib.fsmgen_fill.restype = None
        lib.fsmgen_fill.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64]
        lib.fsmgen_html_block.restype = None
        lib.fsmgen_html_block.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64]
        lib.fsmgen_ac_block.restype = None
        lib.fsmgen_ac_block.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                        ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint32]
        lib.fsmgen_huffman.restype = ctypes.c_uint64
        lib.fsmgen_huffman.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p,
                                       ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p]
        _host = lib
    return _host


def dev_lib() -> ctypes.CDLL:
    global _dev
    if _dev is None:
        lib = ctypes.CDLL(build_dev())
        lib.fsmgen_dev_fill.restype = ctypes.c_int
        lib.fsmgen_dev_fill.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64,
                                        ctypes.c_uint64, ctypes.c_void_p]
        lib.fsmgen_dev_read_stream.restype = ctypes.c_int
        lib.fsmgen_dev_read_stream.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int,
                                               ctypes.c_void_p]
        _dev = lib
    return _dev
