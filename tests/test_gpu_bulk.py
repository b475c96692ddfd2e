"""GPU parity of the bulk runtime operations (steps a9-a16) through the C-ABI
against the CPU oracle: bit-exact on every byte, including bytes the
operation must NOT touch."""
import ctypes

import numpy as np
import pytest

from paper_conf_sc_kimdjjl15_b200 import cl, synth

pytestmark = pytest.mark.gpu


def _rand_bytes(g, n):
    return g.integers(0, 256, n, dtype=np.uint8)


def _copy_rect_gpu(S, src_host, dst_host, so, do, region, srp, ssp, drp, dsp, same=False):
    sb = S.buffer(src_host.nbytes, src_host)
    db = sb if same else S.buffer(dst_host.nbytes, dst_host)
    st = cl.lib().clEnqueueCopyBufferRect(S.queue, sb, db, cl.sz3(so), cl.sz3(do), cl.sz3(region),
                                          srp, ssp, drp, dsp, 0, None, None)
    cl.check(st, "clEnqueueCopyBufferRect")
    out = S.read(db, dst_host.nbytes if not same else src_host.nbytes)
    S.release(sb)
    if not same:
        S.release(db)
    return out


def test_copy_buffer_rect_random_boxes(sess, orc):
    g = synth.rng(30)
    for it in range(150):
        so, do, region, srp, ssp, drp, dsp = synth.random_rect(
            g, max_region=(int(g.choice([7, 64, 300, 5000])), 9, 3), max_pad=(33, 3, 2))
        src = _rand_bytes(g, ssp * (so[2] + region[2]) + 17)
        dst = _rand_bytes(g, dsp * (do[2] + region[2]) + 29)
        got = _copy_rect_gpu(sess, src, dst, so, do, region, srp, ssp, drp, dsp)
        exp = dst.copy()
        orc.copy_rect(src, exp, so, do, region, srp, ssp, drp, dsp)
        assert np.array_equal(got, exp), (it, so, do, region, srp, ssp, drp, dsp)


def test_copy_buffer_rect_staged_long_rows(sess, orc):
    """Misaligned copies with rows >= 2 KiB take the bulk-async staged kernel (16 KiB
    destination chunks): rows around and across chunk boundaries, destination
    alignment constant per row or varying (odd pitches), bytes outside the box kept."""
    g = synth.rng(36)
    cases = [(16384, 3, 0), (16383, 5, 1), (16385, 1, 15), (32768 + 5, 7, 3), (2048, 9, 2),
             (40000, 15, 8), (16384 - 7, 8, 0)]
    for it, (r0, sx, dx) in enumerate(cases):
        for odd_pitch in (False, True):
            region = (r0, int(g.integers(1, 6)), int(g.integers(1, 4)))
            srp = r0 + sx + int(g.integers(0, 40))
            drp = r0 + dx + (int(g.integers(1, 30)) if odd_pitch else 16 * int(g.integers(0, 3)))
            ssp = srp * (region[1] + int(g.integers(0, 3)))
            dsp = drp * (region[1] + int(g.integers(0, 3)))
            so, do = (sx, int(g.integers(0, 2)), 0), (dx, 0, int(g.integers(0, 2)))
            src = _rand_bytes(g, ssp * (so[2] + region[2]) + srp * 2 + 64)
            dst = _rand_bytes(g, dsp * (do[2] + region[2]) + drp * 2 + 64)
            got = _copy_rect_gpu(sess, src, dst, so, do, region, srp, ssp, drp, dsp)
            exp = dst.copy()
            orc.copy_rect(src, exp, so, do, region, srp, ssp, drp, dsp)
            assert np.array_equal(got, exp), (it, odd_pitch, so, do, region, srp, ssp, drp, dsp)


def test_config1_buffer_rect_all_x_origins(sess, orc):
    """BASELINE config 1 (reading A19): region {64 B, 16, 4} out of a 64x64x4 RGBA8
    volume (row pitch 256, slice pitch 16384), every x origin 0..192, also {16 B,16,4}."""
    g = synth.rng(31)
    vol = _rand_bytes(g, 256 * 64 * 4)
    for r0 in (64, 16):
        for x in range(0, 193):
            so = (x, int(g.integers(0, 48)), int(g.integers(0, 1)))
            region = (r0, 16, 4)
            dst = np.zeros((r0 + 7) * 16 * 4 + 64, np.uint8)
            do = (x % 7, 0, 0)
            got = _copy_rect_gpu(sess, vol, dst, so, do, region, 256, 16384, r0 + 7, (r0 + 7) * 16)
            exp = dst.copy()
            orc.copy_rect(vol, exp, so, do, region, 256, 16384, r0 + 7, (r0 + 7) * 16)
            assert np.array_equal(got, exp), (r0, x)


def test_copy_buffer_rect_same_buffer_disjoint(sess, orc):
    g = synth.rng(32)
    buf = _rand_bytes(g, 64 * 8 * 3)
    so, do, region = (0, 0, 0), (32, 0, 0), (32, 8, 3)
    got = _copy_rect_gpu(sess, buf, buf, so, do, region, 64, 512, 64, 512, same=True)
    exp = buf.copy()
    orc.copy_rect(buf.copy(), exp, so, do, region, 64, 512, 64, 512)
    assert np.array_equal(got, exp)
    # overlap is rejected before anything is enqueued
    sb = sess.buffer(buf.nbytes, buf)
    st = cl.lib().clEnqueueCopyBufferRect(sess.queue, sb, sb, cl.sz3((0, 0, 0)), cl.sz3((16, 0, 0)),
                                          cl.sz3(region), 64, 512, 64, 512, 0, None, None)
    assert st == -8
    assert np.array_equal(sess.read(sb, buf.nbytes), buf)
    sess.release(sb)


def test_copy_buffer_large_misaligned(sess):
    g = synth.rng(33)
    n = (1 << 22) + 13
    src = _rand_bytes(g, n)
    sb = sess.buffer(n, src)
    db = sess.buffer(n + 64, np.zeros(n + 64, np.uint8))
    for so, do, size in ((0, 0, n), (3, 5, n - 100), (17, 0, n - 17), (1, 33, 1000), (0, 1, 15)):
        cl.check(cl.lib().clEnqueueCopyBuffer(sess.queue, sb, db, so, do, size, 0, None, None))
        got = sess.read(db, n + 64)
        assert np.array_equal(got[do:do + size], src[so:so + size]), (so, do, size)
    sess.release(sb, db)


@pytest.mark.parametrize("p", [1, 2, 4, 8, 16, 32, 64, 128])
def test_fill_buffer(sess, orc, p):
    g = synth.rng(34 + p)
    n = 1 << 16
    init = _rand_bytes(g, n)
    pat = _rand_bytes(g, p)
    b = sess.buffer(n, init)
    for off, size in ((0, n), (p, 37 * p), (128 * p, 3 * p), (n - 5 * p, 5 * p), (11 * p, 1000 * p)):
        if off + size > n:
            continue
        cl.check(cl.lib().clEnqueueFillBuffer(sess.queue, b, pat.ctypes.data_as(ctypes.c_void_p), p,
                                              off, size, 0, None, None))
        orc.fill_buffer(init, pat.tobytes(), off, size)
        assert np.array_equal(sess.read(b, n), init), (p, off, size)
    sess.release(b)


def test_fill_buffer_on_unaligned_device_pointer(sess, orc):
    """Pattern phase follows the fill start even when the buffer wraps device memory at
    an odd address (b2clCreateBufferFromDevicePointer)."""
    g = synth.rng(35)
    base = sess.buffer(4096, np.zeros(4096, np.uint8))
    ptr = ctypes.c_void_p()
    cl.check(cl.lib().b2clGetMemDevicePointer(base, sess.device, ctypes.byref(ptr)))
    err = ctypes.c_int32()
    sub = cl.lib().b2clCreateBufferFromDevicePointer(sess.ctx, sess.device, 1, ptr.value + 8, 2048,
                                                     ctypes.byref(err))
    cl.check(err.value)
    pat = _rand_bytes(g, 64)
    cl.check(cl.lib().clEnqueueFillBuffer(sess.queue, sub, pat.ctypes.data_as(ctypes.c_void_p), 64,
                                          64, 1024, 0, None, None))
    exp = np.zeros(4096, np.uint8)
    orc.fill_buffer(exp, pat.tobytes(), 8 + 64, 1024)
    assert np.array_equal(sess.read(base, 4096), exp)
    sess.release(sub, base)


IMG_FORMATS = [(cl.CL_RGBA, cl.CL_UNORM_INT8), (cl.CL_RGBA, cl.CL_FLOAT), (cl.CL_R, cl.CL_HALF_FLOAT),
               (cl.CL_RG, cl.CL_SIGNED_INT16), (cl.CL_BGRA, cl.CL_UNORM_INT8), (cl.CL_R, cl.CL_UNSIGNED_INT8),
               (cl.CL_RGBA, cl.CL_UNSIGNED_INT32), (cl.CL_RGB, cl.CL_UNORM_SHORT_565),
               (cl.CL_RGBx, cl.CL_UNORM_INT_101010)]


def _img_pair(S, orc, order, type_, W, H, D, dims, seed):
    g = synth.rng(seed)
    codes = synth.image_codes(g, order, type_, W, H, D)
    img = S.image(order, type_, W, H if dims > 1 else 0, D if dims > 2 else 0, host=codes)
    return img, orc.Image(codes.copy(), W, H, D, dims=dims, order=order, type=type_), codes


@pytest.mark.parametrize("order,type_", IMG_FORMATS)
def test_image_copies_and_fill(sess, orc, order, type_):
    W, H, D = 37, 11, 5
    a, oa, _ = _img_pair(sess, orc, order, type_, W, H, D, 3, 40)
    b, ob, _ = _img_pair(sess, orc, order, type_, W, H, D, 3, 41)
    c2, oc2, _ = _img_pair(sess, orc, order, type_, 29, 13, 1, 2, 42)
    es = orc.elem_size(order, type_)
    L = cl.lib()
    # CopyImage 3D -> 3D, and 3D -> 2D (region[2] = 1)
    cl.check(L.clEnqueueCopyImage(sess.queue, a, b, cl.sz3((3, 2, 1)), cl.sz3((5, 0, 2)),
                                  cl.sz3((20, 9, 3)), 0, None, None))
    orc.copy_image(oa, ob, (3, 2, 1), (5, 0, 2), (20, 9, 3))
    cl.check(L.clEnqueueCopyImage(sess.queue, a, c2, cl.sz3((1, 1, 4)), cl.sz3((2, 3, 0)),
                                  cl.sz3((25, 10, 1)), 0, None, None))
    orc.copy_image(oa, oc2, (1, 1, 4), (2, 3, 0), (25, 10, 1))
    # CopyImageToBuffer / CopyBufferToImage with odd offsets
    nb = 7 + 17 * 6 * 2 * es
    buf = sess.buffer(nb + 16, np.full(nb + 16, 0xAB, np.uint8))
    cl.check(L.clEnqueueCopyImageToBuffer(sess.queue, b, buf, cl.sz3((4, 3, 2)), cl.sz3((17, 6, 2)),
                                          7, 0, None, None))
    hb = np.full(nb + 16, 0xAB, np.uint8)
    orc.copy_image_to_buffer(ob, hb, (4, 3, 2), (17, 6, 2), 7)
    assert np.array_equal(sess.read(buf, nb + 16), hb)
    cl.check(L.clEnqueueCopyBufferToImage(sess.queue, buf, a, 7, cl.sz3((0, 4, 0)),
                                          cl.sz3((17, 6, 2)), 0, None, None))
    orc.copy_buffer_to_image(hb, oa, 7, (0, 4, 0), (17, 6, 2))
    # FillImage with float4 / int4 / uint4 colour
    if type_ in (cl.CL_UNSIGNED_INT8, cl.CL_UNSIGNED_INT32):
        col, rt = np.array([7, 300, 70000, 1], np.uint32), orc.RT_UI
    elif type_ == cl.CL_SIGNED_INT16:
        col, rt = np.array([-7, 40000, -40000, 1], np.int32), orc.RT_I
    else:
        col, rt = np.array([0.25, 1.5, -0.5, 0.7071], np.float32), orc.RT_F
    cl.check(L.clEnqueueFillImage(sess.queue, c2, col.ctypes.data_as(ctypes.c_void_p),
                                  cl.sz3((3, 2, 0)), cl.sz3((20, 7, 1)), 0, None, None))
    orc.fill_image(oc2, rt, col, (3, 2, 0), (20, 7, 1))
    for img, oimg, (w, h, d) in ((a, oa, (W, H, D)), (b, ob, (W, H, D)), (c2, oc2, (29, 13, 1))):
        got = sess.read_image(img, (0, 0, 0), (w, h, d))
        assert np.array_equal(got, oimg.data[:got.size]), (hex(order), hex(type_))
    sess.release(a, b, c2, buf)


def test_read_write_image_host_pitches(sess, orc):
    g = synth.rng(43)
    W, H, D = 19, 7, 4
    img, oimg, _ = _img_pair(sess, orc, cl.CL_RGBA, cl.CL_UNORM_INT16, W, H, D, 3, 43)
    rp, sp = 8 * 12 + 5, (8 * 12 + 5) * 5 + 3
    host = _rand_bytes(g, sp * 3)
    L = cl.lib()
    cl.check(L.clEnqueueWriteImage(sess.queue, img, 1, cl.sz3((4, 1, 1)), cl.sz3((12, 5, 3)), rp, sp,
                                   host.ctypes.data_as(ctypes.c_void_p), 0, None, None))
    orc.write_image_rect(oimg, (4, 1, 1), (12, 5, 3), rp, sp, host)
    rp2, sp2 = 15 * 8 + 9, (15 * 8 + 9) * 6 + 11
    out = np.zeros(sp2 * 3, np.uint8)
    exp = np.zeros(sp2 * 3, np.uint8)
    cl.check(L.clEnqueueReadImage(sess.queue, img, 1, cl.sz3((2, 0, 0)), cl.sz3((15, 6, 3)), rp2,
                                  sp2, out.ctypes.data_as(ctypes.c_void_p), 0, None, None))
    orc.read_image_rect(oimg, (2, 0, 0), (15, 6, 3), rp2, sp2, exp)
    assert np.array_equal(out, exp)
    sess.release(img)


def test_created_contents_visible_to_the_first_command(sess):
    """clCreateBuffer / clCreateImage with host data: the upload has landed
    before the call returns, so the queue's first command (its own stream)
    sees the contents -- a pageable cudaMemcpy returns once the data is
    staged, before its DMA completes (a race seen once in
    test_read_write_buffer_rect before the fix)."""
    g = synth.rng(45)
    L = cl.lib()
    for k in range(12):
        n = (8 << 20) + 16 * k
        host = _rand_bytes(g, n)
        ref = host.copy()
        b = sess.buffer(n, host)
        host[:] = 0  # (the host copy changes right after creation)
        out = np.empty(n, np.uint8)
        cl.check(L.clEnqueueReadBuffer(sess.queue, b, 1, 0, n, out.ctypes.data_as(ctypes.c_void_p), 0, None, None))
        assert np.array_equal(out, ref), k
        sess.release(b)
    W, H = 1024, 512
    codes = synth.image_codes(g, cl.CL_RGBA, cl.CL_FLOAT, W, H)
    img = sess.image(cl.CL_RGBA, cl.CL_FLOAT, W, H, host=codes.copy())
    got = sess.read_image(img, (0, 0, 0), (W, H, 1))
    assert np.array_equal(got.view(np.uint8).reshape(-1), np.ascontiguousarray(codes).view(np.uint8).reshape(-1))
    sess.release(img)


def test_read_write_buffer_rect(sess, orc):
    g = synth.rng(44)
    n = 64 * 10 * 4
    dev_init = _rand_bytes(g, n)
    b = sess.buffer(n, dev_init)
    host = _rand_bytes(g, 50 * 12 * 3)
    L = cl.lib()
    cl.check(L.clEnqueueWriteBufferRect(sess.queue, b, 1, cl.sz3((3, 1, 1)), cl.sz3((5, 2, 0)),
                                        cl.sz3((31, 7, 2)), 64, 640, 50, 600,
                                        host.ctypes.data_as(ctypes.c_void_p), 0, None, None))
    orc.copy_rect(host, dev_init, (5, 2, 0), (3, 1, 1), (31, 7, 2), 50, 600, 64, 640)
    out = np.zeros(n, np.uint8)
    cl.check(L.clEnqueueReadBufferRect(sess.queue, b, 1, cl.sz3((0, 0, 0)), cl.sz3((0, 0, 0)),
                                       cl.sz3((64, 10, 4)), 64, 640, 64, 640,
                                       out.ctypes.data_as(ctypes.c_void_p), 0, None, None))
    assert np.array_equal(out, dev_init)
    sess.release(b)


def test_migrate_same_device_listed_twice(orc):
    """A context with cuda:0 listed twice (two queues, one GPU): migration and
    cross-queue events keep the data equal (reading A24 / O9)."""
    S = cl.Session(0, devices=[0, 0])
    q2 = S.queue_for(0)
    g = synth.rng(45)
    data = _rand_bytes(g, 1 << 20)
    b = S.buffer(data.nbytes, data)
    ev = ctypes.c_void_p()
    L = cl.lib()
    mems = (ctypes.c_void_p * 1)(b)
    cl.check(L.clEnqueueMigrateMemObjects(q2, 1, mems, 0, 0, None, ctypes.byref(ev)))
    out = np.zeros_like(data)
    evs = (ctypes.c_void_p * 1)(ev)
    cl.check(L.clEnqueueReadBuffer(S.queue, b, 1, 0, data.nbytes, out.ctypes.data_as(ctypes.c_void_p),
                                   1, evs, None))
    assert np.array_equal(out, data)
    L.clReleaseEvent(ev)
    L.clReleaseCommandQueue(q2)
    S.release(b)
    S.close()


def test_events_profiling_and_launch_count(orc):
    S = cl.Session(0, profiling=True)
    b = S.buffer(1 << 24)
    pat = np.array([1, 2, 3, 4], np.uint8)
    ev = ctypes.c_void_p()
    L = cl.lib()
    before = cl.launch_count()
    cl.check(L.clEnqueueFillBuffer(S.queue, b, pat.ctypes.data_as(ctypes.c_void_p), 4, 0, 1 << 24, 0,
                                   None, ctypes.byref(ev)))
    evs = (ctypes.c_void_p * 1)(ev)
    cl.check(L.clWaitForEvents(1, evs))
    assert cl.launch_count() == before + 1
    t0, t1 = ctypes.c_uint64(), ctypes.c_uint64()
    cl.check(L.clGetEventProfilingInfo(ev, cl.CL_PROFILING_COMMAND_START, 8, ctypes.byref(t0), None))
    cl.check(L.clGetEventProfilingInfo(ev, cl.CL_PROFILING_COMMAND_END, 8, ctypes.byref(t1), None))
    assert t1.value >= t0.value
    st = ctypes.c_int32()
    cl.check(L.clGetEventInfo(ev, 0x11D3, 4, ctypes.byref(st), None))
    assert st.value == 0
    L.clReleaseEvent(ev)
    S.release(b)
    S.close()


def test_validation_has_no_side_effects(sess):
    g = synth.rng(46)
    data = _rand_bytes(g, 4096)
    b = sess.buffer(4096, data)
    L = cl.lib()
    pat = np.zeros(3, np.uint8)
    assert L.clEnqueueFillBuffer(sess.queue, b, pat.ctypes.data_as(ctypes.c_void_p), 3, 0, 9, 0, None,
                                 None) == -30
    assert L.clEnqueueCopyBufferRect(sess.queue, b, b, cl.sz3((0, 0, 0)), cl.sz3((0, 0, 0)),
                                     cl.sz3((4096, 2, 1)), 0, 0, 0, 0, 0, None, None) == -30
    img = sess.image(cl.CL_RGBA, cl.CL_FLOAT, 8, 8)
    smp = sess.sampler(False, cl.CL_ADDRESS_CLAMP, cl.CL_FILTER_LINEAR)
    assert L.b2clEnqueueReadImageSamples(sess.queue, img, smp, cl.B2CL_RTYPE_UINT, 0, b, 0, 1, b, 0,
                                         0, None, None) == -59                     # A7
    uimg = sess.image(cl.CL_RGBA, cl.CL_UNSIGNED_INT8, 8, 8)
    assert L.b2clEnqueueReadImageSamples(sess.queue, uimg, smp, cl.B2CL_RTYPE_UINT, 0, b, 0, 1, b, 0,
                                         0, None, None) == -59                     # A6
    assert np.array_equal(sess.read(b, 4096), data)
    sess.release(b, img, uimg)
    cl.lib().clReleaseSampler(smp)


def test_config4_full_size_sampled(sess, orc):
    """BASELINE config 4 at full size, in the launch configuration bench.py
    times: the 8 GiB pitched CopyBufferRect (region {16384 B, 2048, 256}, source
    row pitch 16512, slice pitch 2056 * 16512, tight destination), its
    misaligned variant (source origin x = 3, pitch 16387) and the 8 GiB
    FillBuffer; every byte of sampled rows (first / middle / last slices and
    rows, both ragged ends) against the oracle applied to those rows."""
    region = (16384, 2048, 256)
    srp, ssp = 16512, 2056 * 16512
    nsrc = ssp * region[2]
    S_bytes = region[0] * region[1] * region[2]
    src = sess.buffer(nsrc)
    # seeded source contents, one slice at a time (the host never holds 8 GiB)
    for z in range(region[2]):
        sess.write(src, _rand_bytes(synth.rng(4000 + z), ssp), offset=z * ssp)
    dst = sess.buffer(S_bytes)
    zero = cl.sz3((0, 0, 0))
    samples = [(z, y) for z in (0, 1, 127, 253, 254, 255) for y in (0, 1, 1023, 2046, 2047)]

    def src_row(off, n):
        z, r = divmod(off, ssp)
        full = _rand_bytes(synth.rng(4000 + z), ssp)
        row = full[r:r + n]
        if len(row) < n:  # the row continues into the next slice
            row = np.concatenate([row, _rand_bytes(synth.rng(4001 + z), ssp)[:n - len(row)]])
        return row

    def check_rows(so, rp, sp, drp, dsp, reg):
        R0 = reg[0]
        for z, y in samples:
            if z >= reg[2] or y >= reg[1]:
                continue
            s_off = so + z * sp + y * rp
            exp = np.zeros(R0, np.uint8)
            orc.copy_rect(src_row(s_off, R0), exp, (0, 0, 0), (0, 0, 0), (R0, 1, 1), R0, R0, R0, R0)
            got = sess.read(dst, R0, offset=z * dsp + y * drp)
            assert np.array_equal(got, exp), (so, z, y)

    cl.check(cl.lib().clEnqueueCopyBufferRect(sess.queue, src, dst, zero, zero, cl.sz3(region), srp, ssp,
                                              0, 0, 0, None, None))
    check_rows(0, srp, ssp, region[0], region[0] * region[1], region)
    reg2 = (16384, 2048, 255)
    cl.check(cl.lib().clEnqueueCopyBufferRect(sess.queue, src, dst, cl.sz3((3, 0, 0)), zero, cl.sz3(reg2), 16387,
                                              16387 * 2056, 0, 0, 0, None, None))
    check_rows(3, 16387, 16387 * 2056, reg2[0], reg2[0] * reg2[1], reg2)
    pat = np.arange(16, dtype=np.uint8)
    cl.check(cl.lib().clEnqueueFillBuffer(sess.queue, dst, pat.ctypes.data, 16, 0, S_bytes, 0, None, None))
    for off in (0, S_bytes // 2 - 4096, S_bytes - 8192):
        exp = np.zeros(8192, np.uint8)
        orc.fill_buffer(exp, pat.tobytes(), 0, 8192)
        assert np.array_equal(sess.read(dst, 8192, offset=off), exp), off
    sess.release(src, dst)


def test_engine_reference_paths(sess, orc):
    """b2clEnqueueCopyBufferRectEngine / FillBufferEngine (the copy-engine
    references of config 4) give the oracle's bytes, like the SM kernels."""
    L = cl.lib()
    g = synth.rng(321)
    for so, do, region, srp, ssp, drp, dsp in [synth.random_rect(g) for _ in range(6)] + [
            ((0, 0, 0), (0, 0, 0), (64, 8, 3), 80, 80 * 9, 64, 64 * 8)]:
        src = g.integers(0, 256, ssp * (so[2] + region[2]) + 64, dtype=np.uint8)
        dst = g.integers(0, 256, dsp * (do[2] + region[2]) + 64, dtype=np.uint8)
        sb, db = sess.buffer(src.nbytes, src), sess.buffer(dst.nbytes, dst)
        cl.check(L.b2clEnqueueCopyBufferRectEngine(sess.queue, sb, db, cl.sz3(so), cl.sz3(do), cl.sz3(region),
                                                   srp, ssp, drp, dsp, 0, None, None))
        exp = dst.copy()
        orc.copy_rect(src, exp, so, do, region, srp, ssp, drp, dsp)
        assert np.array_equal(sess.read(db, dst.nbytes), exp)
        sess.release(sb, db)
    buf = np.zeros(4096, np.uint8)
    b = sess.buffer(buf.nbytes, buf)
    for ps in (1, 2, 4):
        pat = g.integers(0, 256, ps, dtype=np.uint8)
        cl.check(L.b2clEnqueueFillBufferEngine(sess.queue, b, pat.ctypes.data, ps, 8 * ps, 1000 * ps, 0, None, None))
        orc.fill_buffer(buf, pat.tobytes(), 8 * ps, 1000 * ps)
        assert np.array_equal(sess.read(b, buf.nbytes), buf)
    pat = np.arange(8, dtype=np.uint8)
    assert L.b2clEnqueueFillBufferEngine(sess.queue, b, pat.ctypes.data, 8, 0, 64, 0, None, None) == -30
    sess.release(b)
