"""CPU tests of the C-ABI library: it loads, exports every symbol the headers
declare, and its pure host validators return the Khronos error codes
(pin P8); the rect-overlap test agrees with the oracle's
brute-force byte sets (pin P7).  No compute call is made here."""
import ctypes
import os
import re

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl, synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADERS = [os.path.join(ROOT, "include", h) for h in ("b2cl_cl.h", "b2cl_ext.h")]


@pytest.fixture(scope="module")
def L():
    from paper_conf_sc_kimdjjl15_b200 import build
    build.build()
    return cl.lib()


def declared_functions():
    names = []
    for h in HEADERS:
        src = open(h).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        names += re.findall(r"\b((?:cl|b2cl)[A-Z]\w*)\s*\(", src)
    return sorted(set(names))


def test_every_declared_symbol_is_exported(L):
    names = declared_functions()
    assert len(names) >= 60
    for n in names:
        assert hasattr(L, n), n
    # and the binding declares a prototype for each
    assert set(names) == set(cl.PROTOTYPES), set(names) ^ set(cl.PROTOTYPES)


def test_platform_query_without_gpu(L):
    plat = ctypes.c_void_p()
    num = ctypes.c_uint32()
    assert L.clGetPlatformIDs(1, ctypes.byref(plat), ctypes.byref(num)) == 0
    assert num.value == 1 and plat.value
    buf = ctypes.create_string_buffer(64)
    assert L.clGetPlatformInfo(plat, 0x0902, 64, buf, None) == 0
    assert buf.value == b"b2cl"
    import torch
    if not torch.cuda.is_available():
        n = ctypes.c_uint32()
        assert L.clGetDeviceIDs(plat, cl.CL_DEVICE_TYPE_GPU, 0, None, ctypes.byref(n)) == -1
    assert L.clGetDeviceIDs(plat, 2, 0, None, None) == -30  # no num_devices and no devices


def test_invalid_handles_rejected(L):
    assert L.clFinish(ctypes.c_void_p(0)) == -36
    assert L.clReleaseMemObject(ctypes.c_void_p(0)) == -38
    assert L.clReleaseSampler(ctypes.c_void_p(0)) == -41
    err = ctypes.c_int32()
    assert L.clCreateBuffer(ctypes.c_void_p(0), 1, 16, None, ctypes.byref(err)) is None
    assert err.value == -34


# ---------------------------------------------------------------- P8 error table
RECT_CASES = [
    # (src_size, dst_size, same, so, do, region, srp, ssp, drp, dsp, expected)
    (4096, 4096, 0, (0, 0, 0), (0, 0, 0), (16, 4, 2), 0, 0, 0, 0, 0),
    (4096, 4096, 0, (0, 0, 0), (0, 0, 0), (0, 4, 2), 0, 0, 0, 0, -30),       # zero region
    (4096, 4096, 0, (0, 0, 0), (0, 0, 0), (16, 4, 2), 8, 0, 0, 0, -30),      # row pitch < region[0]
    (4096, 4096, 0, (0, 0, 0), (0, 0, 0), (16, 4, 2), 16, 48, 0, 0, -30),    # slice < region[1]*rp
    (4096, 4096, 0, (0, 0, 0), (0, 0, 0), (16, 4, 2), 16, 72, 0, 0, -30),    # slice % rp != 0
    (4096, 100, 0, (0, 0, 0), (0, 0, 0), (16, 4, 2), 0, 0, 0, 0, 28),        # placeholder (dst OOB)
    (128, 4096, 0, (0, 0, 1), (0, 0, 0), (16, 4, 2), 0, 0, 0, 0, -30),       # src OOB
    (4096, 4096, 1, (0, 0, 0), (16, 0, 0), (16, 4, 2), 32, 128, 32, 128, 0),  # interleaved, no overlap
    (4096, 4096, 1, (0, 0, 0), (8, 0, 0), (16, 4, 2), 32, 128, 32, 128, -8),  # overlap
    (4096, 4096, 1, (0, 0, 0), (0, 0, 1), (16, 4, 2), 32, 128, 64, 256, -30),  # same buffer, pitches differ
    (4096, 4096, 1, (0, 0, 0), (0, 0, 2), (16, 4, 2), 32, 128, 32, 128, 0),   # disjoint slices
]


@pytest.mark.parametrize("case", RECT_CASES)
def test_p8_copy_buffer_rect_errors(L, case):
    ss, ds, same, so, do, region, srp, ssp, drp, dsp, exp = case
    if exp == 28:
        exp = -30
    got = L.b2clValidateCopyBufferRect(ss, ds, same, cl.sz3(so), cl.sz3(do), cl.sz3(region),
                                       srp, ssp, drp, dsp)
    assert got == exp


def test_p7_overlap_matches_oracle_bruteforce(L, orc):
    g = synth.rng(20)
    n_overlap = 0
    for _ in range(3000):
        region = [int(g.integers(1, 9)), int(g.integers(1, 5)), int(g.integers(1, 4))]
        rp = region[0] + int(g.integers(0, 9))
        sp = rp * (region[1] + int(g.integers(0, 3)))
        so = [int(g.integers(0, 12)), int(g.integers(0, 5)), int(g.integers(0, 3))]
        do = [int(g.integers(0, 12)), int(g.integers(0, 5)), int(g.integers(0, 3))]
        exp = orc.rect_overlap(so, do, region, rp, sp, rp, sp)
        got = L.b2clRectOverlap(cl.sz3(so), cl.sz3(do), cl.sz3(region), rp, sp)
        assert bool(got) == exp, (so, do, region, rp, sp)
        n_overlap += exp
    assert 300 < n_overlap < 2700  # both outcomes well represented


@pytest.mark.parametrize("size,ps,off,n,exp", [
    (1024, 4, 0, 1024, 0), (1024, 3, 0, 12, -30), (1024, 256, 0, 256, -30), (1024, 0, 0, 0, -30),
    (1024, 8, 4, 16, -30), (1024, 8, 8, 12, -30), (1024, 8, 1016, 16, -30), (1024, 128, 896, 128, 0),
    (1024, 1, 1023, 1, 0), (1024, 16, 0, 0, 0)])
def test_p8_fill_buffer_errors(L, size, ps, off, n, exp):
    assert L.b2clValidateFillBuffer(size, ps, off, n) == exp


def test_p8_sampler_errors(L):
    ok = 0
    for norm in (0, 1, 2):
        for am in range(0x112F, 0x1136):
            for fm in (0x1139, 0x1140, 0x1141):
                got = L.b2clValidateSampler(norm, am, fm)
                valid = (norm in (0, 1) and 0x1130 <= am <= 0x1134 and fm in (0x1140, 0x1141)
                         and (norm == 1 or am <= 0x1132))
                assert got == (0 if valid else -30), (norm, am, fm)
                ok += valid
    assert ok == 16  # the 16 valid samplers (8 address/normalization combos x 2 filters)


def _layout(L, order, type_, itype, w, h=0, d=0, mips=0):
    fmt = cl.ImageFormat(order, type_)
    desc = cl.ImageDesc(itype, w, h, d, 0, 0, 0, mips, 0, None)
    es, rp, sp, tot = (ctypes.c_size_t() for _ in range(4))
    st = L.b2clImageLayout(ctypes.byref(fmt), ctypes.byref(desc), ctypes.byref(es),
                           ctypes.byref(rp), ctypes.byref(sp), ctypes.byref(tot))
    return st, es.value, rp.value, sp.value, tot.value


def test_image_layout_and_format_errors(L, orc):
    I2, I3, I1 = cl.CL_MEM_OBJECT_IMAGE2D, cl.CL_MEM_OBJECT_IMAGE3D, cl.CL_MEM_OBJECT_IMAGE1D
    assert _layout(L, cl.CL_RGBA, cl.CL_FLOAT, I2, 4096, 4096) == (0, 16, 65536, 65536 * 4096,
                                                                   65536 * 4096 * 1)
    assert _layout(L, cl.CL_R, cl.CL_FLOAT, I3, 512, 512, 512)[:4] == (0, 4, 2048, 2048 * 512)
    assert _layout(L, cl.CL_RGBA, cl.CL_UNORM_INT8, I2, 65, 33)[:3] == (0, 4, 384)
    assert _layout(L, cl.CL_RGB, cl.CL_UNORM_INT8, I2, 4, 4)[0] == -10       # RGB: packed only
    assert _layout(L, cl.CL_BGRA, cl.CL_FLOAT, I2, 4, 4)[0] == -10
    assert _layout(L, cl.CL_RGBA, 0x10D4, I2, 4, 4)[0] == -10                # packed 565
    assert _layout(L, 0x1234, cl.CL_FLOAT, I2, 4, 4)[0] == -39
    assert _layout(L, cl.CL_RGBA, cl.CL_FLOAT, I2, 0, 4)[0] == -65
    assert _layout(L, cl.CL_RGBA, cl.CL_FLOAT, I2, 70000, 4)[0] == -40
    assert _layout(L, cl.CL_RGBA, cl.CL_FLOAT, 0x10F3, 4, 4)[0] == -65       # 2D array: NEXT(2)
    assert _layout(L, cl.CL_RGBA, cl.CL_FLOAT, I2, 4, 4, mips=1)[0] == -65
    assert _layout(L, cl.CL_R, cl.CL_HALF_FLOAT, I1, 100)[:3] == (0, 2, 256)
    # element sizes agree with the oracle's table for every (order, type) it supports
    for o in range(0x10B0, 0x10BA):
        for t in range(0x10D0, 0x10DF):
            st, es = _layout(L, o, t, I2, 3, 3)[:2]
            oes = orc.elem_size(o, t)
            assert (st == 0) == (oes > 0), (hex(o), hex(t))
            if st == 0:
                assert es == oes


@pytest.mark.parametrize("itype,dims,o,r,exp", [
    (cl.CL_MEM_OBJECT_IMAGE2D, (8, 4, 1), (0, 0, 0), (8, 4, 1), 0),
    (cl.CL_MEM_OBJECT_IMAGE2D, (8, 4, 1), (0, 0, 1), (8, 4, 1), -30),
    (cl.CL_MEM_OBJECT_IMAGE2D, (8, 4, 1), (0, 0, 0), (8, 4, 2), -30),
    (cl.CL_MEM_OBJECT_IMAGE2D, (8, 4, 1), (1, 0, 0), (8, 4, 1), -30),
    (cl.CL_MEM_OBJECT_IMAGE2D, (8, 4, 1), (0, 0, 0), (0, 4, 1), -30),
    (cl.CL_MEM_OBJECT_IMAGE1D, (8, 1, 1), (0, 1, 0), (8, 1, 1), -30),
    (cl.CL_MEM_OBJECT_IMAGE3D, (8, 4, 3), (7, 3, 2), (1, 1, 1), 0),
    (cl.CL_MEM_OBJECT_IMAGE3D, (8, 4, 3), (7, 3, 2), (1, 1, 2), -30),
])
def test_p8_image_box_errors(L, itype, dims, o, r, exp):
    assert L.b2clValidateImageBox(itype, *dims, cl.sz3(o), cl.sz3(r)) == exp


def test_binding_fails_loudly_without_library(monkeypatch, tmp_path):
    monkeypatch.setattr(cl, "LIB_PATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(cl, "_lib", None)
    with pytest.raises(RuntimeError, match="no CPU fallback"):
        cl.lib()


# ---------------------------------------------------------------- texture mapping (row 3)
def _map(L, stored_order, stored_type, modes, filt, rmode, norm, dims, border=(0, 0, 0, 0)):
    td = cl.texture_desc(modes, filt, rmode, norm, border)
    st = cl.ImageFormat(stored_order, stored_type)
    view = cl.ImageFormat()
    nc, am, fm, rt = ctypes.c_uint32(), ctypes.c_uint32(), ctypes.c_uint32(), ctypes.c_uint32()
    r = L.b2clTextureMapping(ctypes.byref(td), dims, ctypes.byref(st), ctypes.byref(view),
                             ctypes.byref(nc), ctypes.byref(am), ctypes.byref(fm), ctypes.byref(rt))
    return r, (view.image_channel_order, view.image_channel_data_type), nc.value, am.value, fm.value, rt.value


def test_texture_mapping_table(L, orc):
    """The CUDA texture -> (image view, sampler) mapping of P:449 (reading A40): the
    same table the oracle's translation pin (tests/test_oracle_cuda_tex.py) proves exact."""
    from tests.test_oracle_cuda_tex import CL_ADDR, CL_FILT, _cl_type
    stored = [cl.CL_UNSIGNED_INT8, cl.CL_SIGNED_INT8, cl.CL_UNSIGNED_INT16, cl.CL_SIGNED_INT16,
              cl.CL_UNSIGNED_INT32, cl.CL_SIGNED_INT32, cl.CL_HALF_FLOAT, cl.CL_FLOAT,
              cl.CL_UNORM_INT8, cl.CL_SNORM_INT16]
    n = 0
    for t in stored:
        for rmode in (0, 1):
            for mode in range(4):
                for filt in (0, 1):
                    for norm in (False, True):
                        r, view, nc, am, fm, rt = _map(L, cl.CL_RGBA, t, [mode] * 2, filt, rmode, norm, 2)
                        # what the oracle side expects
                        raw = {cl.CL_UNORM_INT8: cl.CL_UNSIGNED_INT8, cl.CL_SNORM_INT16: cl.CL_SIGNED_INT16}.get(t, t)
                        bits32_or_float = raw in (cl.CL_UNSIGNED_INT32, cl.CL_SIGNED_INT32, cl.CL_HALF_FLOAT, cl.CL_FLOAT)
                        if rmode == 1 and bits32_or_float:
                            assert r == -30, (hex(t), rmode)
                            continue
                        if not norm and mode in (0, 2):
                            assert r == -30
                            continue
                        ctype, ort = _cl_type(orc, raw, rmode)
                        if filt == 1 and ort != orc.RT_F:
                            assert r == -59
                            continue
                        assert r == 0, (hex(t), rmode, mode, filt, norm, r)
                        assert view == (cl.CL_RGBA, ctype) and rt == ort
                        assert (nc, am, fm) == (int(norm), CL_ADDR[mode], CL_FILT[filt])
                        n += 1
    assert n > 100
    # per-axis modes must agree on the sampled axes only
    assert _map(L, cl.CL_R, cl.CL_FLOAT, [1, 3], 0, 0, True, 2)[0] == -30
    assert _map(L, cl.CL_R, cl.CL_FLOAT, [1, 3], 0, 0, True, 1)[0] == 0
    assert _map(L, cl.CL_R, cl.CL_FLOAT, [1, 1, 3], 0, 0, True, 2)[0] == 0
    # border colour other than 0, orders and packed types CUDA textures do not have
    assert _map(L, cl.CL_R, cl.CL_FLOAT, [3], 0, 0, True, 1, border=(0, 0, 0, 1))[0] == -30
    assert _map(L, cl.CL_BGRA, cl.CL_UNORM_INT8, [1], 0, 1, True, 1)[0] == -10
    assert _map(L, cl.CL_RGB, cl.CL_UNORM_SHORT_565, [1], 0, 1, True, 1)[0] == -10


def test_channel_format_desc(L):
    def fmt(x, y, z, w, kind):
        d = cl.ChannelFormatDesc(x, y, z, w, kind)
        f = cl.ImageFormat()
        r = L.b2clChannelFormat(ctypes.byref(d), ctypes.byref(f))
        return r, (f.image_channel_order, f.image_channel_data_type)
    S, U, F = cl.B2CL_CHANNEL_SIGNED, cl.B2CL_CHANNEL_UNSIGNED, cl.B2CL_CHANNEL_FLOAT
    assert fmt(8, 8, 8, 8, U) == (0, (cl.CL_RGBA, cl.CL_UNSIGNED_INT8))
    assert fmt(16, 0, 0, 0, S) == (0, (cl.CL_R, cl.CL_SIGNED_INT16))
    assert fmt(32, 32, 0, 0, F) == (0, (cl.CL_RG, cl.CL_FLOAT))
    assert fmt(16, 16, 16, 16, F) == (0, (cl.CL_RGBA, cl.CL_HALF_FLOAT))
    assert fmt(32, 0, 0, 0, U) == (0, (cl.CL_R, cl.CL_UNSIGNED_INT32))
    for bad in ((8, 8, 8, 0, U), (8, 16, 0, 0, U), (0, 8, 0, 0, U), (8, 0, 8, 0, U), (8, 0, 0, 0, F),
                (64, 0, 0, 0, S), (8, 0, 0, 0, 7)):
        assert fmt(*bad)[0] == -10, bad
