"""Thin ctypes binding of libb2cl.so: the same names as include/b2cl_cl.h and
include/b2cl_ext.h, argument marshalling only.  Every step of the hot path
runs in the library's CUDA kernels; there is no Python or CPU fallback:
if the library is missing, the first call raises.

`Session` is a small convenience layer (one context + one queue on a device,
numpy in / numpy out) used by the tests, smoke() and bench.py.  It calls
only the C-ABI functions below.
"""
from __future__ import annotations

import ctypes
import os
from ctypes import POINTER, byref, c_float, c_int32, c_size_t, c_uint32, c_uint64, c_void_p

import numpy as np

LIB_PATH = os.environ.get("B2CL_LIB") or os.path.join(os.path.dirname(os.path.abspath(__file__)),
                                                    "libb2cl.so")  # B2CL_LIB: A/B builds

# ---- Khronos / b2cl constants (restated from include/*.h) ----
CL_SUCCESS = 0
CL_DEVICE_TYPE_GPU = 1 << 2
CL_DEVICE_TYPE_ALL = 0xFFFFFFFF
CL_QUEUE_PROFILING_ENABLE = 1 << 1
CL_MEM_READ_WRITE, CL_MEM_WRITE_ONLY, CL_MEM_READ_ONLY = 1, 2, 4
CL_MEM_USE_HOST_PTR, CL_MEM_ALLOC_HOST_PTR, CL_MEM_COPY_HOST_PTR = 8, 16, 32
B2CL_MEM_IPC_EXPORTABLE = 1 << 40
B2CL_MEM_TILED_IMAGE = 1 << 41
CL_MEM_OBJECT_BUFFER, CL_MEM_OBJECT_IMAGE2D, CL_MEM_OBJECT_IMAGE3D = 0x10F0, 0x10F1, 0x10F2
CL_MEM_OBJECT_IMAGE2D_ARRAY, CL_MEM_OBJECT_IMAGE1D = 0x10F3, 0x10F4
CL_MEM_OBJECT_IMAGE1D_ARRAY, CL_MEM_OBJECT_IMAGE1D_BUFFER = 0x10F5, 0x10F6
CL_R, CL_A, CL_RG, CL_RA, CL_RGB, CL_RGBA, CL_BGRA, CL_ARGB, CL_INTENSITY, CL_LUMINANCE = range(0x10B0, 0x10BA)
CL_SNORM_INT8, CL_SNORM_INT16, CL_UNORM_INT8, CL_UNORM_INT16 = 0x10D0, 0x10D1, 0x10D2, 0x10D3
CL_SIGNED_INT8, CL_SIGNED_INT16, CL_SIGNED_INT32 = 0x10D7, 0x10D8, 0x10D9
CL_UNSIGNED_INT8, CL_UNSIGNED_INT16, CL_UNSIGNED_INT32 = 0x10DA, 0x10DB, 0x10DC
CL_HALF_FLOAT, CL_FLOAT = 0x10DD, 0x10DE
CL_Rx, CL_RGx, CL_RGBx = 0x10BA, 0x10BB, 0x10BC
CL_UNORM_SHORT_565, CL_UNORM_SHORT_555, CL_UNORM_INT_101010 = 0x10D4, 0x10D5, 0x10D6
CL_ADDRESS_NONE, CL_ADDRESS_CLAMP_TO_EDGE, CL_ADDRESS_CLAMP, CL_ADDRESS_REPEAT, \
    CL_ADDRESS_MIRRORED_REPEAT = range(0x1130, 0x1135)
CL_FILTER_NEAREST, CL_FILTER_LINEAR = 0x1140, 0x1141
CL_MIGRATE_MEM_OBJECT_HOST, CL_MIGRATE_MEM_OBJECT_CONTENT_UNDEFINED = 1, 2
CL_IMAGE_FORMAT, CL_IMAGE_ELEMENT_SIZE, CL_IMAGE_ROW_PITCH, CL_IMAGE_SLICE_PITCH = 0x1110, 0x1111, 0x1112, 0x1113
CL_IMAGE_WIDTH, CL_IMAGE_HEIGHT, CL_IMAGE_DEPTH = 0x1114, 0x1115, 0x1116
CL_IMAGE_ARRAY_SIZE, CL_IMAGE_BUFFER = 0x1117, 0x1118
CL_PROFILING_COMMAND_START, CL_PROFILING_COMMAND_END = 0x1282, 0x1283
B2CL_RTYPE_FLOAT, B2CL_RTYPE_INT, B2CL_RTYPE_UINT = 0, 1, 2
B2CL_COORD_FLOAT, B2CL_COORD_INT = 0, 1
# CUDA texture front end (b2cl_ext.h): cudaResourceDesc / cudaTextureDesc values
B2CL_RESOURCE_ARRAY, B2CL_RESOURCE_LINEAR, B2CL_RESOURCE_PITCH2D = 0, 2, 3
B2CL_CHANNEL_SIGNED, B2CL_CHANNEL_UNSIGNED, B2CL_CHANNEL_FLOAT = 0, 1, 2
B2CL_TEX_WRAP, B2CL_TEX_CLAMP, B2CL_TEX_MIRROR, B2CL_TEX_BORDER = 0, 1, 2, 3
B2CL_TEX_POINT, B2CL_TEX_LINEAR = 0, 1
B2CL_READ_ELEMENT_TYPE, B2CL_READ_NORMALIZED_FLOAT = 0, 1

_H = c_void_p
_P = c_void_p
_S = c_size_t
_I = c_int32
_U = c_uint32
_L = c_uint64
_SZ3 = POINTER(c_size_t)
_PI = POINTER(c_int32)

# name -> (restype, argtypes); covers every entry point of include/*.h
PROTOTYPES = {
    "clGetPlatformIDs": (_I, [_U, POINTER(_H), POINTER(_U)]),
    "clGetPlatformInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clGetDeviceIDs": (_I, [_H, _L, _U, POINTER(_H), POINTER(_U)]),
    "clGetDeviceInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clCreateContext": (_H, [_P, _U, POINTER(_H), _P, _P, _PI]),
    "clRetainContext": (_I, [_H]),
    "clReleaseContext": (_I, [_H]),
    "clGetContextInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clCreateCommandQueue": (_H, [_H, _H, _L, _PI]),
    "clRetainCommandQueue": (_I, [_H]),
    "clReleaseCommandQueue": (_I, [_H]),
    "clGetCommandQueueInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clFlush": (_I, [_H]),
    "clFinish": (_I, [_H]),
    "clCreateBuffer": (_H, [_H, _L, _S, _P, _PI]),
    "clCreateImage": (_H, [_H, _L, _P, _P, _P, _PI]),
    "clGetSupportedImageFormats": (_I, [_H, _L, _U, _U, _P, POINTER(_U)]),
    "clRetainMemObject": (_I, [_H]),
    "clReleaseMemObject": (_I, [_H]),
    "clGetMemObjectInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clGetImageInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clCreateSampler": (_H, [_H, _U, _U, _U, _PI]),
    "clRetainSampler": (_I, [_H]),
    "clReleaseSampler": (_I, [_H]),
    "clGetSamplerInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clWaitForEvents": (_I, [_U, POINTER(_H)]),
    "clRetainEvent": (_I, [_H]),
    "clReleaseEvent": (_I, [_H]),
    "clGetEventInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clGetEventProfilingInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clEnqueueMarkerWithWaitList": (_I, [_H, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueBarrierWithWaitList": (_I, [_H, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueReadBuffer": (_I, [_H, _H, _U, _S, _S, _P, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueWriteBuffer": (_I, [_H, _H, _U, _S, _S, _P, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueReadBufferRect": (_I, [_H, _H, _U, _SZ3, _SZ3, _SZ3, _S, _S, _S, _S, _P, _U,
                                     POINTER(_H), POINTER(_H)]),
    "clEnqueueWriteBufferRect": (_I, [_H, _H, _U, _SZ3, _SZ3, _SZ3, _S, _S, _S, _S, _P, _U,
                                      POINTER(_H), POINTER(_H)]),
    "clEnqueueCopyBuffer": (_I, [_H, _H, _H, _S, _S, _S, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueCopyBufferRect": (_I, [_H, _H, _H, _SZ3, _SZ3, _SZ3, _S, _S, _S, _S, _U,
                                     POINTER(_H), POINTER(_H)]),
    "clEnqueueFillBuffer": (_I, [_H, _H, _P, _S, _S, _S, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueReadImage": (_I, [_H, _H, _U, _SZ3, _SZ3, _S, _S, _P, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueWriteImage": (_I, [_H, _H, _U, _SZ3, _SZ3, _S, _S, _P, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueCopyImage": (_I, [_H, _H, _H, _SZ3, _SZ3, _SZ3, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueFillImage": (_I, [_H, _H, _P, _SZ3, _SZ3, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueCopyImageToBuffer": (_I, [_H, _H, _H, _SZ3, _SZ3, _S, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueCopyBufferToImage": (_I, [_H, _H, _H, _S, _SZ3, _SZ3, _U, POINTER(_H), POINTER(_H)]),
    "clEnqueueMigrateMemObjects": (_I, [_H, _U, POINTER(_H), _L, _U, POINTER(_H), POINTER(_H)]),
    "clCreateProgramWithBinary": (_H, [_H, _U, POINTER(_H), POINTER(_S), _P, _PI, _PI]),
    "clBuildProgram": (_I, [_H, _U, POINTER(_H), ctypes.c_char_p, _P, _P]),
    "clGetProgramBuildInfo": (_I, [_H, _H, _U, _S, _P, POINTER(_S)]),
    "clRetainProgram": (_I, [_H]),
    "clReleaseProgram": (_I, [_H]),
    "clCreateKernel": (_H, [_H, ctypes.c_char_p, _PI]),
    "clRetainKernel": (_I, [_H]),
    "clReleaseKernel": (_I, [_H]),
    "clGetKernelInfo": (_I, [_H, _U, _S, _P, POINTER(_S)]),
    "clSetKernelArg": (_I, [_H, _U, _S, _P]),
    "clEnqueueNDRangeKernel": (_I, [_H, _H, _U, _SZ3, _SZ3, _SZ3, _U, POINTER(_H), POINTER(_H)]),
    "b2clEnqueueReadImageSamples": (_I, [_H, _H, _H, _U, _U, _H, _S, _S, _H, _S, _U, POINTER(_H),
                                         POINTER(_H)]),
    "b2clEnqueueReadImageGrid": (_I, [_H, _H, _H, _U, POINTER(c_float), _SZ3, _U, _H, _S, _U,
                                      POINTER(_H), POINTER(_H)]),
    "b2clEnqueueReadImageGridRegion": (_I, [_H, _H, _H, _U, POINTER(c_float), _SZ3, _SZ3, _U, _H,
                                            _S, _U, POINTER(_H), POINTER(_H)]),
    "b2clCreateImageShard": (_H, [_H, _L, _P, _P, _S, _S, _S, _P, _PI]),
    "b2clEnqueueWriteImageSamples": (_I, [_H, _H, _U, _H, _S, _S, _H, _S, _U, POINTER(_H),
                                          POINTER(_H)]),
    "b2clCreateCommandQueueWithStream": (_H, [_H, _H, _P, _L, _PI]),
    "b2clGetCommandQueueStream": (_I, [_H, POINTER(_P)]),
    "b2clGetDeviceOrdinal": (_I, [_H, _PI]),
    "b2clSetAllocator": (_I, [_P, _P]),
    "b2clCreateBufferFromDevicePointer": (_H, [_H, _H, _L, _P, _S, _PI]),
    "b2clGetMemDevicePointer": (_I, [_H, _H, POINTER(_P)]),
    "b2clGetMemIpcHandle": (_I, [_H, _P]),
    "b2clCreateBufferFromIpcHandle": (_H, [_H, _H, _P, _S, _PI]),
    "b2clCreateImageFromIpcHandle": (_H, [_H, _H, _L, _P, _P, _P, _PI]),
    "b2clEnqueueCopyBufferEngine": (_I, [_H, _H, _H, _S, _S, _S, _U, POINTER(_H), POINTER(_H)]),
    "b2clEnqueueCopyBufferRectEngine": (_I, [_H, _H, _H, _SZ3, _SZ3, _SZ3, _S, _S, _S, _S, _U,
                                             POINTER(_H), POINTER(_H)]),
    "b2clEnqueueFillBufferEngine": (_I, [_H, _H, _P, _S, _S, _S, _U, POINTER(_H), POINTER(_H)]),
    "b2clGetKernelLaunchCount": (_L, []),
    "b2clGetLastKernelName": (ctypes.c_char_p, []),
    "b2clValidateCopyBufferRect": (_I, [_S, _S, _I, _SZ3, _SZ3, _SZ3, _S, _S, _S, _S]),
    "b2clRectOverlap": (_I, [_SZ3, _SZ3, _SZ3, _S, _S]),
    "b2clValidateFillBuffer": (_I, [_S, _S, _S, _S]),
    "b2clValidateSampler": (_I, [_U, _U, _U]),
    "b2clImageLayout": (_I, [_P, _P, POINTER(_S), POINTER(_S), POINTER(_S), POINTER(_S)]),
    "b2clValidateImageBox": (_I, [_U, _S, _S, _S, _SZ3, _SZ3]),
    "b2clCreateTextureObject": (_I, [_H, _P, _P, _P]),
    "b2clDestroyTextureObject": (_I, [_P]),
    "b2clTextureMapping": (_I, [_P, _U, _P, _P, POINTER(_U), POINTER(_U), POINTER(_U), POINTER(_U)]),
    "b2clChannelFormat": (_I, [_P, _P]),
}


class ImageFormat(ctypes.Structure):
    _fields_ = [("image_channel_order", c_uint32), ("image_channel_data_type", c_uint32)]


class ImageDesc(ctypes.Structure):
    _fields_ = [("image_type", c_uint32), ("image_width", c_size_t), ("image_height", c_size_t),
                ("image_depth", c_size_t), ("image_array_size", c_size_t),
                ("image_row_pitch", c_size_t), ("image_slice_pitch", c_size_t),
                ("num_mip_levels", c_uint32), ("num_samples", c_uint32), ("buffer", c_void_p)]


class ChannelFormatDesc(ctypes.Structure):  # b2cl_channel_format_desc
    _fields_ = [("x", c_int32), ("y", c_int32), ("z", c_int32), ("w", c_int32), ("kind", c_uint32)]


class ResourceDesc(ctypes.Structure):  # b2cl_resource_desc
    _fields_ = [("res_type", c_uint32), ("mem", c_void_p), ("offset", c_size_t),
                ("desc", ChannelFormatDesc), ("size_in_bytes", c_size_t), ("width", c_size_t),
                ("height", c_size_t), ("pitch_in_bytes", c_size_t)]


class TextureDesc(ctypes.Structure):  # b2cl_texture_desc
    _fields_ = [("address_mode", c_uint32 * 3), ("filter_mode", c_uint32), ("read_mode", c_uint32),
                ("normalized_coords", c_int32), ("border_color", c_float * 4)]


class Texture(ctypes.Structure):  # b2cl_texture
    _fields_ = [("image", c_void_p), ("sampler", c_void_p), ("rtype", c_uint32)]


def texture_desc(address_modes, filter_mode: int, read_mode: int, normalized: bool,
                 border=(0.0, 0.0, 0.0, 0.0)) -> TextureDesc:
    am = list(address_modes) + [B2CL_TEX_WRAP] * (3 - len(address_modes))
    return TextureDesc((c_uint32 * 3)(*am[:3]), filter_mode, read_mode, int(bool(normalized)),
                       (c_float * 4)(*border))


class CLError(RuntimeError):
    def __init__(self, code: int, what: str = ""):
        super().__init__(f"{what} failed with OpenCL error {code}")
        self.code = code


_lib = None


def lib():
    """Load libb2cl.so (raises if it was not built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: build it with "
                               "`python -m paper_conf_sc_kimdjjl15_b200.build` (no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in PROTOTYPES.items():
            f = getattr(L, name, None)
            if f is None:  # an older A/B build (B2CL_LIB); the ABI test checks the real one
                continue
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def __getattr__(name):  # cl.clFinish(...) etc. resolve to the C function
    if name in PROTOTYPES:
        return getattr(lib(), name)
    raise AttributeError(name)


def check(code: int, what: str = "") -> None:
    if code != CL_SUCCESS:
        raise CLError(code, what)


def sz3(v) -> ctypes.Array:
    v = [int(x) for x in v]
    v = v + [0] * (3 - len(v)) if len(v) < 3 else v[:3]
    return (c_size_t * 3)(*v)


def _ptr(a: np.ndarray) -> c_void_p:
    return c_void_p(a.ctypes.data)


def launch_count() -> int:
    return int(lib().b2clGetKernelLaunchCount())


def last_kernel() -> str:
    """The kernel the library's last launch from this thread used."""
    return lib().b2clGetLastKernelName().decode()


# ---- torch allocator hook (device memory from PyTorch's caching allocator) ----
_ALLOC_T = ctypes.CFUNCTYPE(c_void_p, c_size_t, ctypes.c_int, c_void_p)
_FREE_T = ctypes.CFUNCTYPE(None, c_void_p, ctypes.c_int, c_void_p)
_hooks = []


def use_torch_allocator() -> None:
    import torch

    def _alloc(size, device, stream):
        try:
            return torch.cuda.caching_allocator_alloc(int(size), int(device), stream or None)
        except Exception:  # allocation failure -> NULL -> CL_MEM_OBJECT_ALLOCATION_FAILURE
            return None

    def _free(ptr, device, stream):
        torch.cuda.caching_allocator_delete(int(ptr))

    a, f = _ALLOC_T(_alloc), _FREE_T(_free)
    _hooks[:] = [a, f]
    check(lib().b2clSetAllocator(ctypes.cast(a, c_void_p), ctypes.cast(f, c_void_p)),
          "b2clSetAllocator")


def default_allocator() -> None:
    check(lib().b2clSetAllocator(None, None), "b2clSetAllocator")


# =============================================================== Session
class Session:
    """One context + one in-order queue on CUDA device `device_index`
    (index among the platform's devices)."""

    def __init__(self, device_index: int = 0, stream: int | None = None, profiling: bool = False,
                 devices=None):
        L = lib()
        plat = c_void_p()
        check(L.clGetPlatformIDs(1, byref(plat), None), "clGetPlatformIDs")
        n = c_uint32()
        check(L.clGetDeviceIDs(plat, CL_DEVICE_TYPE_GPU, 0, None, byref(n)), "clGetDeviceIDs")
        devs = (c_void_p * n.value)()
        check(L.clGetDeviceIDs(plat, CL_DEVICE_TYPE_GPU, n.value, devs, None), "clGetDeviceIDs")
        self.all_devices = list(devs)
        ctx_devs = [self.all_devices[i] for i in (devices or [device_index])]
        err = c_int32()
        arr = (c_void_p * len(ctx_devs))(*ctx_devs)
        self.ctx = L.clCreateContext(None, len(ctx_devs), arr, None, None, byref(err))
        check(err.value, "clCreateContext")
        self.device = self.all_devices[device_index]
        props = CL_QUEUE_PROFILING_ENABLE if profiling else 0
        if stream is None:
            self.queue = L.clCreateCommandQueue(self.ctx, self.device, props, byref(err))
        else:
            self.queue = L.b2clCreateCommandQueueWithStream(self.ctx, self.device, c_void_p(stream),
                                                            props, byref(err))
        check(err.value, "clCreateCommandQueue")
        self._objs = []

    def queue_for(self, device_index: int, profiling: bool = False):
        err = c_int32()
        q = lib().clCreateCommandQueue(self.ctx, self.all_devices[device_index],
                                       CL_QUEUE_PROFILING_ENABLE if profiling else 0, byref(err))
        check(err.value, "clCreateCommandQueue")
        return q

    def stream(self) -> int:
        s = c_void_p()
        check(lib().b2clGetCommandQueueStream(self.queue, byref(s)), "b2clGetCommandQueueStream")
        return s.value or 0

    def ordinal(self) -> int:
        o = c_int32()
        check(lib().b2clGetDeviceOrdinal(self.device, byref(o)), "b2clGetDeviceOrdinal")
        return o.value

    # ---- objects ----
    def buffer(self, nbytes: int, host: np.ndarray | None = None, flags: int = CL_MEM_READ_WRITE):
        err = c_int32()
        if host is not None:
            host = np.ascontiguousarray(host)
            flags |= CL_MEM_COPY_HOST_PTR
            m = lib().clCreateBuffer(self.ctx, flags, int(nbytes), _ptr(host), byref(err))
        else:
            m = lib().clCreateBuffer(self.ctx, flags, int(nbytes), None, byref(err))
        check(err.value, "clCreateBuffer")
        return m

    def image(self, order: int, type_: int, width: int, height: int = 0, depth: int = 0,
              host: np.ndarray | None = None, host_row_pitch: int = 0, host_slice_pitch: int = 0,
              flags: int = CL_MEM_READ_WRITE):
        dims = 3 if depth else (2 if height else 1)
        fmt = ImageFormat(order, type_)
        desc = ImageDesc({1: CL_MEM_OBJECT_IMAGE1D, 2: CL_MEM_OBJECT_IMAGE2D,
                          3: CL_MEM_OBJECT_IMAGE3D}[dims], width, height, depth, 0,
                         host_row_pitch, host_slice_pitch, 0, 0, None)
        err = c_int32()
        if host is not None:
            host = np.ascontiguousarray(host)
            m = lib().clCreateImage(self.ctx, flags | CL_MEM_COPY_HOST_PTR, byref(fmt), byref(desc),
                                    _ptr(host), byref(err))
        else:
            m = lib().clCreateImage(self.ctx, flags, byref(fmt), byref(desc), None, byref(err))
        check(err.value, "clCreateImage")
        return m

    def image_array(self, order: int, type_: int, width: int, layers: int, height: int = 0,
                    host: np.ndarray | None = None, host_row_pitch: int = 0,
                    host_slice_pitch: int = 0, flags: int = CL_MEM_READ_WRITE):
        """A 1D image array (height 0) or 2D image array of `layers` layers."""
        fmt = ImageFormat(order, type_)
        desc = ImageDesc(CL_MEM_OBJECT_IMAGE2D_ARRAY if height else CL_MEM_OBJECT_IMAGE1D_ARRAY,
                         width, height, 0, layers, host_row_pitch, host_slice_pitch, 0, 0, None)
        err = c_int32()
        if host is not None:
            host = np.ascontiguousarray(host)
            m = lib().clCreateImage(self.ctx, flags | CL_MEM_COPY_HOST_PTR, byref(fmt), byref(desc),
                                    _ptr(host), byref(err))
        else:
            m = lib().clCreateImage(self.ctx, flags, byref(fmt), byref(desc), None, byref(err))
        check(err.value, "clCreateImage (array)")
        return m

    def image_buffer(self, order: int, type_: int, width: int, buffer, flags: int = 0):
        """A 1D image buffer over `buffer`'s bytes (CL_MEM_OBJECT_IMAGE1D_BUFFER)."""
        fmt = ImageFormat(order, type_)
        desc = ImageDesc(CL_MEM_OBJECT_IMAGE1D_BUFFER, width, 0, 0, 0, 0, 0, 0, 0, buffer)
        err = c_int32()
        m = lib().clCreateImage(self.ctx, flags, byref(fmt), byref(desc), None, byref(err))
        check(err.value, "clCreateImage (1D buffer)")
        return m

    def image_shard(self, order: int, type_: int, width: int, height: int, depth: int,
                    begin: int, count: int, halo: int = 0, host: np.ndarray | None = None,
                    flags: int = CL_MEM_READ_WRITE):
        """Rows [begin, begin+count) (+halo) of a global width x height (x depth) image;
        `host` holds the stored rows/slices, tightly packed."""
        dims = 3 if depth else 2
        fmt = ImageFormat(order, type_)
        desc = ImageDesc(CL_MEM_OBJECT_IMAGE3D if dims == 3 else CL_MEM_OBJECT_IMAGE2D, width,
                         height, depth, 0, 0, 0, 0, 0, None)
        err = c_int32()
        if host is not None:
            host = np.ascontiguousarray(host)
            m = lib().b2clCreateImageShard(self.ctx, flags | CL_MEM_COPY_HOST_PTR, byref(fmt),
                                           byref(desc), begin, count, halo, _ptr(host), byref(err))
        else:
            m = lib().b2clCreateImageShard(self.ctx, flags, byref(fmt), byref(desc), begin, count,
                                           halo, None, byref(err))
        check(err.value, "b2clCreateImageShard")
        return m

    def texture(self, res: ResourceDesc, tex_desc: TextureDesc) -> Texture:
        """b2clCreateTextureObject: the (image view, sampler) pair of a CUDA texture."""
        t = Texture()
        check(lib().b2clCreateTextureObject(self.ctx, byref(res), byref(tex_desc), byref(t)),
              "b2clCreateTextureObject")
        return t

    def sampler(self, normalized: bool, addressing: int, filt: int):
        err = c_int32()
        s = lib().clCreateSampler(self.ctx, int(bool(normalized)), addressing, filt, byref(err))
        check(err.value, "clCreateSampler")
        return s

    def image_info(self, img, name: int) -> int:
        v = c_size_t()
        check(lib().clGetImageInfo(img, name, ctypes.sizeof(v), byref(v), None), "clGetImageInfo")
        return v.value

    # ---- transfers ----
    def write(self, buf, host: np.ndarray, offset: int = 0, blocking: bool = True) -> None:
        host = np.ascontiguousarray(host)
        check(lib().clEnqueueWriteBuffer(self.queue, buf, int(blocking), offset, host.nbytes,
                                         _ptr(host), 0, None, None), "clEnqueueWriteBuffer")

    def read(self, buf, nbytes: int, dtype=np.uint8, offset: int = 0) -> np.ndarray:
        out = np.empty(nbytes, dtype=np.uint8)
        check(lib().clEnqueueReadBuffer(self.queue, buf, 1, offset, nbytes, _ptr(out), 0, None,
                                        None), "clEnqueueReadBuffer")
        return out.view(dtype)

    def read_image(self, img, origin, region, row_pitch=0, slice_pitch=0, nbytes=None):
        es = self.image_info(img, CL_IMAGE_ELEMENT_SIZE)
        rp = row_pitch or region[0] * es
        sp = slice_pitch or rp * region[1]
        out = np.zeros(nbytes or sp * region[2], dtype=np.uint8)
        check(lib().clEnqueueReadImage(self.queue, img, 1, sz3(origin), sz3(region), row_pitch,
                                       slice_pitch, _ptr(out), 0, None, None), "clEnqueueReadImage")
        return out

    # ---- programs and kernels (translated kernels, include/b2cl_device.cuh) ----
    def program(self, binary: bytes):
        err = c_int32()
        buf = ctypes.create_string_buffer(binary, len(binary))
        bins = (c_void_p * 1)(ctypes.cast(buf, c_void_p))
        lens = (c_size_t * 1)(len(binary))
        devs = (c_void_p * 1)(self.device)
        prog = lib().clCreateProgramWithBinary(self.ctx, 1, devs, lens, bins, None, byref(err))
        check(err.value, "clCreateProgramWithBinary")
        st = lib().clBuildProgram(prog, 0, None, None, None, None)
        if st != CL_SUCCESS:
            log = ctypes.create_string_buffer(4096)
            lib().clGetProgramBuildInfo(prog, self.device, 0x1183, 4096, log, None)
            raise CLError(st, f"clBuildProgram ({log.value.decode(errors='replace')})")
        return prog

    def kernel(self, prog, name: str):
        err = c_int32()
        k = lib().clCreateKernel(prog, name.encode(), byref(err))
        check(err.value, "clCreateKernel")
        return k

    def set_args(self, k, *args) -> None:
        """Each arg: a handle (c_void_p: cl_mem / cl_sampler), ("local", nbytes), or a
        ctypes scalar (c_int32(3), c_float(2.0), ...)."""
        for i, a in enumerate(args):
            if isinstance(a, tuple) and a[0] == "local":
                st = lib().clSetKernelArg(k, i, int(a[1]), None)
            elif isinstance(a, (int, c_void_p)) and not isinstance(a, bool):
                h = c_void_p(a.value if isinstance(a, c_void_p) else a)
                st = lib().clSetKernelArg(k, i, ctypes.sizeof(h), byref(h))
            else:
                st = lib().clSetKernelArg(k, i, ctypes.sizeof(a), byref(a))
            check(st, f"clSetKernelArg({i})")

    def ndrange(self, k, gws, lws=None, offset=None) -> None:
        dim = len(gws)
        check(lib().clEnqueueNDRangeKernel(self.queue, k, dim, sz3(offset) if offset else None,
                                           sz3(gws), sz3(lws) if lws else None, 0, None, None),
              "clEnqueueNDRangeKernel")

    def finish(self) -> None:
        check(lib().clFinish(self.queue), "clFinish")

    def release(self, *objs) -> None:
        for o in objs:
            lib().clReleaseMemObject(o)

    def close(self) -> None:
        L = lib()
        L.clReleaseCommandQueue(self.queue)
        L.clReleaseContext(self.ctx)
