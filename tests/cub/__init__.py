"""ctypes loader for tests/cub/libcubref.so (CUB DeviceReduce) -- test and bench
context only (SURVEY 8(c) pin P10; the paper's comparison system)."""
import ctypes
import os
import subprocess

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "cub_ref.cu")
_LIB = os.path.join(_HERE, "libcubref.so")
_lib = None


def build(force=False):
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-std=c++17", "-Xcompiler", "-fPIC", "-shared", "-o", _LIB + ".tmp", _SRC])
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        L.cubref_reduce.restype = ctypes.c_int
        L.cubref_reduce.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t,
                                    ctypes.c_void_p, ctypes.c_void_p]
        _lib = L
    return _lib


def reduce(dtype_code, op_code, in_ptr, n, out_ptr, stream=0):
    st = lib().cubref_reduce(dtype_code, op_code, in_ptr or None, n, out_ptr or None, stream or None)
    if st != 0:
        raise RuntimeError(f"cub reduce failed: cudaError {st}")
