"""CPU oracle of the OpenCL 1.2 image / sampler / memory-object rules.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference``) may import
this package.  The product path (``paper_conf_sc_kimdjjl15_b200``) never
imports it, and the two share no code: the C source is ``oracle/oracle.c``
(see its header for the citations to PAPER.md and [CL1.2]).

This module only marshals numpy arrays into the C functions; all arithmetic
is in ``oracle.c``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_HDR = os.path.join(_HERE, "oracle.h")
_LIB = os.path.join(_HERE, "liboracle.so")

# Khronos values restated (oracle.h); kept local so nothing is shared with the product.
R, A, RG, RA, RGB, RGBA, BGRA, ARGB, INTENSITY, LUMINANCE = range(0x10B0, 0x10BA)
SNORM_INT8, SNORM_INT16, UNORM_INT8, UNORM_INT16 = 0x10D0, 0x10D1, 0x10D2, 0x10D3
SIGNED_INT8, SIGNED_INT16, SIGNED_INT32 = 0x10D7, 0x10D8, 0x10D9
UNSIGNED_INT8, UNSIGNED_INT16, UNSIGNED_INT32 = 0x10DA, 0x10DB, 0x10DC
HALF_FLOAT, FLOAT = 0x10DD, 0x10DE
Rx, RGx, RGBx = 0x10BA, 0x10BB, 0x10BC
UNORM_SHORT_565, UNORM_SHORT_555, UNORM_INT_101010 = 0x10D4, 0x10D5, 0x10D6
ADDRESS_NONE, ADDRESS_CLAMP_TO_EDGE, ADDRESS_CLAMP, ADDRESS_REPEAT, ADDRESS_MIRRORED_REPEAT = range(0x1130, 0x1135)
FILTER_NEAREST, FILTER_LINEAR = 0x1140, 0x1141
RT_F, RT_I, RT_UI = 0, 1, 2


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-ffp-contract=off, no fast-math)."""
    if os.environ.get("B2CL_ORACLE_LIB"):
        return os.environ["B2CL_ORACLE_LIB"]
    if (not force and os.path.exists(_LIB)
            and os.path.getmtime(_LIB) >= max(os.path.getmtime(_SRC), os.path.getmtime(_HDR))):
        return _LIB
    tmp = _LIB + f".tmp{os.getpid()}"
    cmd = ["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
           "-shared", "-Wall", "-Wextra", "-Wno-unused-parameter", "-o", tmp, _SRC,
           "-lm", "-lpthread"]
    subprocess.run(cmd, check=True)
    os.replace(tmp, _LIB)
    return _LIB


class _Image(ctypes.Structure):
    _fields_ = [("data", ctypes.c_void_p),
                ("width", ctypes.c_int64), ("height", ctypes.c_int64), ("depth", ctypes.c_int64),
                ("row_pitch", ctypes.c_int64), ("slice_pitch", ctypes.c_int64),
                ("dims", ctypes.c_int32), ("order", ctypes.c_uint32), ("type", ctypes.c_uint32),
                ("arrayed", ctypes.c_int32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        # B2CL_ORACLE_LIB: a prebuilt oracle library (tools/mutate_oracle.py
        # loads deliberately mutated copies through it to prove the pins bite)
        L = ctypes.CDLL(os.environ.get("B2CL_ORACLE_LIB") or build())
        sz3 = ctypes.POINTER(ctypes.c_size_t)
        P = ctypes.c_void_p
        i64, u32, i32 = ctypes.c_int64, ctypes.c_uint32, ctypes.c_int
        L.oracle_elem_size.argtypes = [u32, u32]
        L.oracle_channels.argtypes = [u32]
        L.oracle_half_to_float.argtypes = [ctypes.c_uint16]
        L.oracle_half_to_float.restype = ctypes.c_float
        L.oracle_float_to_half_rte.argtypes = [ctypes.c_float]
        L.oracle_float_to_half_rte.restype = ctypes.c_uint16
        L.oracle_norm_to_float.argtypes = [u32, ctypes.c_int32]
        L.oracle_norm_to_float.restype = ctypes.c_float
        L.oracle_float_to_norm.argtypes = [u32, ctypes.c_float]
        L.oracle_float_to_norm.restype = ctypes.c_int32
        L.oracle_axis_nearest.argtypes = [ctypes.c_float, i64, i32, u32, ctypes.POINTER(i64)]
        L.oracle_axis_linear.argtypes = [ctypes.c_float, i64, i32, u32, ctypes.POINTER(i64),
                                         ctypes.POINTER(i64), ctypes.POINTER(ctypes.c_float)]
        L.oracle_layer_index.argtypes = [ctypes.c_float, i64]
        L.oracle_layer_index.restype = i64
        L.oracle_read_samples.argtypes = [P, i32, u32, u32, i32, i32, P, i64, i64, P]
        L.oracle_read_grid.argtypes = [P, i32, u32, u32, i32, P, i64, i64, i64, i32,
                                       i64, i64, i64, i64, P, i32]
        L.oracle_write_samples.argtypes = [P, i32, P, i64, P, i64]
        L.oracle_convert_texel.argtypes = [u32, u32, i32, P, P]
        L.oracle_tex_fetch.argtypes = [P, P, P, P]
        L.oracle_tex1Dfetch.argtypes = [P, u32, ctypes.c_int32, P]
        L.oracle_copy_rect.argtypes = [P, P, sz3, sz3, sz3, ctypes.c_size_t, ctypes.c_size_t,
                                       ctypes.c_size_t, ctypes.c_size_t]
        L.oracle_copy_rect.restype = None
        L.oracle_fill_buffer.argtypes = [P, P, ctypes.c_size_t, ctypes.c_size_t, ctypes.c_size_t]
        L.oracle_fill_buffer.restype = None
        L.oracle_fill_image.argtypes = [P, i32, P, sz3, sz3]
        L.oracle_copy_image.argtypes = [P, P, sz3, sz3, sz3]
        L.oracle_copy_image.restype = None
        L.oracle_copy_image_to_buffer.argtypes = [P, P, sz3, sz3, ctypes.c_size_t]
        L.oracle_copy_image_to_buffer.restype = None
        L.oracle_copy_buffer_to_image.argtypes = [P, P, ctypes.c_size_t, sz3, sz3]
        L.oracle_copy_buffer_to_image.restype = None
        L.oracle_read_image_rect.argtypes = [P, sz3, sz3, ctypes.c_size_t, ctypes.c_size_t, P]
        L.oracle_read_image_rect.restype = None
        L.oracle_write_image_rect.argtypes = [P, sz3, sz3, ctypes.c_size_t, ctypes.c_size_t, P]
        L.oracle_write_image_rect.restype = None
        L.oracle_rect_overlap.argtypes = [sz3, sz3, sz3, ctypes.c_size_t, ctypes.c_size_t,
                                          ctypes.c_size_t, ctypes.c_size_t]
        _lib = L
    return _lib


def _sz3(v):
    v = list(v) + [0] * (3 - len(v))
    return (ctypes.c_size_t * 3)(*[int(x) for x in v[:3]])


def _ptr(a: np.ndarray) -> ctypes.c_void_p:
    return ctypes.c_void_p(a.ctypes.data)


class Image:
    """A host image for the oracle: a byte array plus the Fig. 6 fields.

    Image arrays: ``arrayed=True`` with ``dims`` the sampled axes (1 or 2); the
    layers are ``height`` (1D array) or ``depth`` (2D array)."""

    def __init__(self, data: np.ndarray, width: int, height: int = 1, depth: int = 1,
                 dims: int = 2, order: int = RGBA, type: int = FLOAT,
                 row_pitch: int = 0, slice_pitch: int = 0, arrayed: bool = False):
        es = elem_size(order, type)
        if es < 0:
            raise ValueError("format not supported")
        self.elem_size = es
        self.row_pitch = row_pitch or width * es
        self.slice_pitch = slice_pitch or self.row_pitch * height
        need = self.slice_pitch * (depth - 1) + self.row_pitch * (height - 1) + width * es
        self.data = np.ascontiguousarray(data).view(np.uint8).reshape(-1)
        if self.data.size < need:
            raise ValueError(f"image data too small: {self.data.size} < {need}")
        self.width, self.height, self.depth, self.dims = width, height, depth, dims
        self.order, self.type = order, type
        self.arrayed = bool(arrayed)
        if self.arrayed and dims not in (1, 2):
            raise ValueError("image arrays are 1D or 2D")

    def cstruct(self) -> _Image:
        return _Image(self.data.ctypes.data, self.width, self.height, self.depth,
                      self.row_pitch, self.slice_pitch, self.dims, self.order, self.type,
                      int(self.arrayed))


def elem_size(order: int, type: int) -> int:
    return lib().oracle_elem_size(order, type)


def _check(st: int) -> None:
    if st != 0:
        raise OracleError(st)


class OracleError(RuntimeError):
    def __init__(self, code: int):
        super().__init__(f"oracle returned {code}")
        self.code = code


def read_samples(img: Image, normalized: bool, addressing: int, filt: int, rtype: int,
                 coords: np.ndarray) -> np.ndarray:
    """read_image{f,i,ui} at each row of coords (float32 or int32, shape (n, c))."""
    coords = np.ascontiguousarray(coords)
    is_int = coords.dtype == np.int32
    if not is_int:
        coords = coords.astype(np.float32, copy=False)
    n = coords.shape[0]
    cstride = coords.shape[1] if coords.ndim > 1 else 1
    out = np.zeros((n, 4), dtype=np.float32 if rtype == RT_F else (np.int32 if rtype == RT_I else np.uint32))
    s = img.cstruct()
    _check(lib().oracle_read_samples(ctypes.byref(s), int(normalized), addressing, filt, rtype,
                                     int(is_int), _ptr(coords), cstride, n, _ptr(out)))
    return out


def read_grid(img: Image, normalized: bool, addressing: int, filt: int, rtype: int,
              affine: np.ndarray, out_dims, out_channels: int,
              zrange=None, yrange=None, nthreads: int = 1) -> np.ndarray:
    A = np.ascontiguousarray(np.asarray(affine, dtype=np.float32).reshape(12))
    w, h, d = (list(out_dims) + [1, 1])[:3]
    z0, z1 = zrange if zrange is not None else (0, d)
    y0, y1 = yrange if yrange is not None else (0, h)
    dt = np.float32 if rtype == RT_F else (np.int32 if rtype == RT_I else np.uint32)
    out = np.zeros((z1 - z0, y1 - y0, w, out_channels), dtype=dt)
    s = img.cstruct()
    _check(lib().oracle_read_grid(ctypes.byref(s), int(normalized), addressing, filt, rtype,
                                  _ptr(A), w, h, d, out_channels, z0, z1, y0, y1,
                                  _ptr(out), nthreads))
    return out


def write_samples(img: Image, rtype: int, icoords: np.ndarray, colors: np.ndarray) -> None:
    icoords = np.ascontiguousarray(icoords, dtype=np.int32)
    colors = np.ascontiguousarray(colors)
    assert colors.itemsize == 4 and colors.size == 4 * icoords.shape[0]
    cstride = icoords.shape[1] if icoords.ndim > 1 else 1
    s = img.cstruct()
    _check(lib().oracle_write_samples(ctypes.byref(s), rtype, _ptr(icoords), cstride,
                                      _ptr(colors), icoords.shape[0]))


def convert_texel(order: int, type: int, rtype: int, color) -> bytes:
    col = np.ascontiguousarray(np.asarray(color)).view(np.uint8)
    assert col.size == 16
    out = np.zeros(16, dtype=np.uint8)
    _check(lib().oracle_convert_texel(order, type, rtype, _ptr(col), _ptr(out)))
    return out[:elem_size(order, type)].tobytes()


# ---- CUDA texture fetches (oracle.h: NEXT row 3) ----
TEX_WRAP, TEX_CLAMP, TEX_MIRROR, TEX_BORDER = 0, 1, 2, 3
TEX_POINT, TEX_LINEAR = 0, 1
TEX_ELEMENT, TEX_NORMALIZED = 0, 1


class _TexDesc(ctypes.Structure):
    _fields_ = [("address_mode", ctypes.c_uint32 * 3), ("filter_mode", ctypes.c_uint32),
                ("read_mode", ctypes.c_uint32), ("normalized_coords", ctypes.c_int32)]


def tex_fetch(img: Image, address_modes, filter_mode: int, read_mode: int, normalized: bool,
              coords: np.ndarray) -> np.ndarray:
    """tex1D/2D/3D (tex*Layered when img.arrayed: the last coordinate is the layer)
    at each row of coords; returns (n, 4) uint32 bit patterns."""
    am = list(address_modes) + [0] * (3 - len(address_modes))
    td = _TexDesc((ctypes.c_uint32 * 3)(*am[:3]), filter_mode, read_mode, int(normalized))
    coords = np.ascontiguousarray(coords, dtype=np.float32)
    n = coords.shape[0]
    out = np.zeros((n, 4), np.uint32)
    s = img.cstruct()
    for k in range(n):
        _check(lib().oracle_tex_fetch(ctypes.byref(s), ctypes.byref(td),
                                      ctypes.c_void_p(coords[k].ctypes.data),
                                      ctypes.c_void_p(out[k].ctypes.data)))
    return out


def tex1Dfetch(img: Image, read_mode: int, xs) -> np.ndarray:
    xs = np.asarray(xs, np.int32)
    out = np.zeros((xs.size, 4), np.uint32)
    s = img.cstruct()
    for k in range(xs.size):
        _check(lib().oracle_tex1Dfetch(ctypes.byref(s), read_mode, int(xs[k]),
                                       ctypes.c_void_p(out[k].ctypes.data)))
    return out


def copy_rect(src: np.ndarray, dst: np.ndarray, src_origin, dst_origin, region,
              src_row_pitch=0, src_slice_pitch=0, dst_row_pitch=0, dst_slice_pitch=0) -> None:
    lib().oracle_copy_rect(_ptr(src), _ptr(dst), _sz3(src_origin), _sz3(dst_origin), _sz3(region),
                           src_row_pitch, src_slice_pitch, dst_row_pitch, dst_slice_pitch)


def fill_buffer(buf: np.ndarray, pattern: bytes, offset: int, size: int) -> None:
    p = np.frombuffer(pattern, dtype=np.uint8).copy()
    lib().oracle_fill_buffer(_ptr(buf), _ptr(p), len(pattern), offset, size)


def fill_image(img: Image, rtype: int, color, origin, region) -> None:
    col = np.ascontiguousarray(np.asarray(color)).view(np.uint8)
    s = img.cstruct()
    _check(lib().oracle_fill_image(ctypes.byref(s), rtype, _ptr(col), _sz3(origin), _sz3(region)))


def copy_image(src: Image, dst: Image, src_origin, dst_origin, region) -> None:
    a, b = src.cstruct(), dst.cstruct()
    lib().oracle_copy_image(ctypes.byref(a), ctypes.byref(b), _sz3(src_origin), _sz3(dst_origin),
                            _sz3(region))


def copy_image_to_buffer(src: Image, dst: np.ndarray, src_origin, region, dst_offset: int) -> None:
    a = src.cstruct()
    lib().oracle_copy_image_to_buffer(ctypes.byref(a), _ptr(dst), _sz3(src_origin), _sz3(region),
                                      dst_offset)


def copy_buffer_to_image(src: np.ndarray, dst: Image, src_offset: int, dst_origin, region) -> None:
    b = dst.cstruct()
    lib().oracle_copy_buffer_to_image(_ptr(src), ctypes.byref(b), src_offset, _sz3(dst_origin),
                                      _sz3(region))


def read_image_rect(img: Image, origin, region, row_pitch, slice_pitch, host: np.ndarray) -> None:
    a = img.cstruct()
    lib().oracle_read_image_rect(ctypes.byref(a), _sz3(origin), _sz3(region), row_pitch,
                                 slice_pitch, _ptr(host))


def write_image_rect(img: Image, origin, region, row_pitch, slice_pitch, host: np.ndarray) -> None:
    a = img.cstruct()
    lib().oracle_write_image_rect(ctypes.byref(a), _sz3(origin), _sz3(region), row_pitch,
                                  slice_pitch, _ptr(host))


def rect_overlap(src_origin, dst_origin, region, srp=0, ssp=0, drp=0, dsp=0) -> bool:
    return bool(lib().oracle_rect_overlap(_sz3(src_origin), _sz3(dst_origin), _sz3(region),
                                          srp, ssp, drp, dsp))


def layer_index(c: float, n: int) -> int:
    """[CL1.2 §8.4] layer = clamp(rint(c), 0, n - 1)."""
    return lib().oracle_layer_index(c, n)


def axis_nearest(s: float, n: int, normalized: bool, addressing: int) -> int:
    i = ctypes.c_int64()
    lib().oracle_axis_nearest(s, n, int(normalized), addressing, ctypes.byref(i))
    return i.value


def axis_linear(s: float, n: int, normalized: bool, addressing: int):
    i0, i1, a = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_float()
    lib().oracle_axis_linear(s, n, int(normalized), addressing, ctypes.byref(i0),
                             ctypes.byref(i1), ctypes.byref(a))
    return i0.value, i1.value, a.value
