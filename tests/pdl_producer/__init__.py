"""ctypes loader for tests/pdl_producer/libproducer.so -- TEST ONLY: a kernel
that triggers its programmatic dependents before writing (see producer.cu)."""
import ctypes
import os
import subprocess

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "producer.cu")
_LIB = os.path.join(_HERE, "libproducer.so")
_lib = None


def build(force=False):
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-Xcompiler", "-fPIC", "-shared", "-o", _LIB + ".tmp", _SRC])
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        L.producer_launch.restype = ctypes.c_int
        L.producer_launch.argtypes = [ctypes.c_void_p, ctypes.c_longlong, ctypes.c_int, ctypes.c_longlong,
                                      ctypes.c_void_p, ctypes.c_int]
        _lib = L
    return _lib


def produce(ptr, n, value, delay_cycles, stream, pdl=True):
    st = lib().producer_launch(ptr, n, value, delay_cycles, stream or None, 1 if pdl else 0)
    if st != 0:
        raise RuntimeError(f"producer launch failed: cudaError {st}")
