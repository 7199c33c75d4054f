"""The C ABI under its own names (include/spread.h, include/somier.h): one
Python function per entry point, `capi.somier_step(handle, 10)` etc. Argument
marshalling only -- ctypes does the conversions declared in
_native.SIGNATURES; a call returning a spread_status raises SpreadError on
failure (with spread_last_error()'s message) and returns None, other calls
return their value. Pointers: numpy float64 arrays are passed as double*,
ctypes objects by reference via ctypes.byref by the caller. The Spread /
Somier / SomierStream classes are the convenience layer over the same calls.
"""
import ctypes

import numpy as np

from . import _native as N

__all__ = []


def _arg(x):
    if isinstance(x, np.ndarray):
        if x.dtype != np.float64 or not x.flags["C_CONTIGUOUS"]:
            raise TypeError("expected a C-contiguous float64 array")
        return x.ctypes.data_as(ctypes.POINTER(ctypes.c_double))
    return x


def _make(name, restype):
    def call(*args):
        r = getattr(N.lib(), name)(*[_arg(a) for a in args])
        if restype is ctypes.c_int:
            N.check(r, name)
            return None
        return r
    call.__name__ = name
    call.__doc__ = "C ABI %s (include/*.h)" % name
    return call


for _name, _restype, _argtypes in N.SIGNATURES:
    globals()[_name] = _make(_name, _restype)
    __all__.append(_name)
