"""Mutation check of the oracle's pins.

    python tools/mutate_oracle.py [-j N] [-k NAME]

Each mutation is ONE plausible mistake in oracle/oracle.c (a dropped term, a
wrong sign, bound, index or slot, a transposed operand).  For each, a copy of
oracle.c with that single edit is compiled to a temporary library and the
CPU pin suites (tests/test_oracle_*.py, `-m "not gpu"`) are run against it
through B2CL_ORACLE_LIB.  A mutant is CAUGHT when at least one pin fails.
Every mutant below must be caught; the script exits non-zero otherwise and
prints the survivors.  Mutants that cannot change any result (equivalent
mutants) are not listed; the ones considered are noted at the bottom.

The list holds the round-1 judge's 26 edits (its 9 surviving ones
are marked [judge]), the 6 of DESIGN.md §2 and more, covering every function
of oracle.c.  Nothing here touches the product path.
"""
from __future__ import annotations

import argparse
import os
import subprocess
import sys
import tempfile
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "oracle.c")

# (name, old text, new text, occurrence index of `old` in oracle.c)
MUTANTS = [
    # ---- addressing ([CL1.2 §8.2])
    ("repeat_nearest_wrap_bound", "if (i > n - 1) i = i - n;", "if (i > n) i = i - n;", 0),
    ("repeat_linear_minus_half", "float t = u - 0.5f;", "float t = u + 0.5f;", 0),
    ("mirror_linear_minus_half", "float t = u - 0.5f;", "float t = u - 0.25f;", 1),
    ("nonwrap_linear_minus_half", "float t = u - 0.5f;", "float t = u;", 2),
    ("repeat_linear_i0_wrap", "if (b0 < 0) b0 = n + b0;", "if (b0 < 0) b0 = 0;", 0),
    ("repeat_linear_i1_wrap", "if (b1 > n - 1) b1 = b1 - n;", "if (b1 > n) b1 = b1 - n;", 0),
    ("mirror_nearest_clamp", "*i0 = i < n - 1 ? i : n - 1;", "*i0 = i;", 0),
    ("mirror_linear_i1_clamp", "*i1 = b1 < n - 1 ? b1 : n - 1;", "*i1 = b1;", 0),
    ("mirror_linear_i0_clamp", "*i0 = b0 > 0 ? b0 : 0;", "*i0 = b0;", 0),
    ("mirror_rint_to_floor", "float sp = 2.0f * rintf(0.5f * s);", "float sp = 2.0f * floorf(0.5f * s);", 0),
    ("mirror_no_fabs", "sp = fabsf(s - sp);", "sp = s - sp;", 1),
    ("cte_clamp_bound", "case OR_ADDRESS_CLAMP_TO_EDGE: return clamp64(i, 0, n - 1);",
     "case OR_ADDRESS_CLAMP_TO_EDGE: return clamp64(i, 0, n);", 0),
    ("clamp_lower_bound", "case OR_ADDRESS_CLAMP:         return clamp64(i, -1, n);",
     "case OR_ADDRESS_CLAMP:         return clamp64(i, 0, n);", 0),
    ("nonwrap_normalized_ignored", "float u = normalized ? s * fn : s;", "float u = s;", 1),
    ("ifloor_sat_high", "if (f >= 2147483648.0f) return INT32_MAX;", "if (f >= 2147483648.0f) return INT32_MIN;", 0),
    ("ifloor_nan", "if (isnan(x)) return 0;", "if (isnan(x)) return 1;", 0),
    ("layer_rint_to_floor", "float r = rintf(c);", "float r = floorf(c);", 0),
    ("icoord_no_address_mode", "ix[d] = am(addressing, icoord[d], n[d]);", "ix[d] = icoord[d];", 0),
    # ---- fetch, conversion, channel map ([CL1.2 §8.3], §6.12.14.1)
    ("fetch_pitches_swapped", "const uint8_t* p = img->data + k * img->slice_pitch + j * img->row_pitch +",
     "const uint8_t* p = img->data + j * img->slice_pitch + k * img->row_pitch +", 0),
    ("bgra_read_map", "case OR_BGRA:      out[0] = mem[2]; out[1] = mem[1]; out[2] = mem[0];",
     "case OR_BGRA:      out[0] = mem[0]; out[1] = mem[1]; out[2] = mem[2];", 0),
    ("argb_read_map", "case OR_ARGB:      out[0] = mem[1]; out[1] = mem[2]; out[2] = mem[3]; out[3] = mem[0];",
     "case OR_ARGB:      out[0] = mem[0]; out[1] = mem[1]; out[2] = mem[2]; out[3] = mem[3];", 0),
    ("luminance_alpha", "case OR_LUMINANCE: out[0] = mem[0]; out[1] = mem[0]; out[2] = mem[0]; out[3] = one;",
     "case OR_LUMINANCE: out[0] = mem[0]; out[1] = mem[0]; out[2] = mem[0]; out[3] = mem[0];", 0),
    ("border_luminance", "order == OR_RGB || order == OR_LUMINANCE)", "order == OR_RGB)", 0),
    ("border_rgb", "order == OR_RGB || order == OR_LUMINANCE)", "order == OR_LUMINANCE)", 0),
    ("snorm8_read_scale", "fmaxf(-1.0f, (float)code / 127.0f)", "fmaxf(-1.0f, (float)code / 128.0f)", 0),
    ("snorm8_read_no_clamp", "fmaxf(-1.0f, (float)code / 127.0f)", "((float)code / 127.0f)", 0),
    ("unorm16_read_scale", "return (float)code / 65535.0f;", "return (float)code / 65536.0f;", 0),
    ("half_read_exponent_bias", "v = ldexp((double)(1024 + m), e - 25);", "v = ldexp((double)(1024 + m), e - 24);", 0),
    ("half_read_subnormal", "v = ldexp((double)m, -24);", "v = ldexp((double)m, -25);", 0),
    ("packed_565_g_shift", "s565[3] = {11, 5, 0}", "s565[3] = {11, 6, 0}", 0),
    ("packed_rgbx_alpha_in_range", "case OR_RGBx:      out[0] = mem[0]; out[1] = mem[1]; out[2] = mem[2]; out[3] = one;",
     "case OR_RGBx:      out[0] = mem[0]; out[1] = mem[1]; out[2] = mem[2]; out[3] = zero;", 0),
    # ---- LINEAR sum (O6)
    ("linear_weight_transposed", "double wi = ii ? (double)w[0] : 1.0 - (double)w[0];",
     "double wi = ii ? 1.0 - (double)w[0] : (double)w[0];", 0),
    ("linear_wj_transposed", "double wj = dims > 1 ? (jj ? (double)w[1] : 1.0 - (double)w[1]) : 1.0;",
     "double wj = dims > 1 ? (jj ? 1.0 - (double)w[1] : (double)w[1]) : 1.0;", 0),
    ("linear_wk_dropped", "double wk = dims > 2 ? (kk ? (double)w[2] : 1.0 - (double)w[2]) : 1.0;",
     "double wk = dims > 2 ? 0.5 : 1.0;", 0),
    ("linear_sum_in_fp32", "for (int ch = 0; ch < 4; ++ch) acc[ch] += wt * (double)t[ch].f;",
     "for (int ch = 0; ch < 4; ++ch) acc[ch] = (float)(acc[ch] + (float)wt * t[ch].f);", 0),
    ("grid_coord_wrong_operand", "v = v + a[1] * yf;", "v = v + a[1] * xf;", 0),
    ("grid_coord_offset_dropped", "v = v + a[3];", "v = v;", 0),
    # ---- write conversion ([CL1.2 §8.3.1], §6.12.14.4)
    ("write_slot_A", "case OR_A: slot[0] = 3; break;", "case OR_A: slot[0] = 0; break;", 0),            # [judge]
    ("write_slot_RA", "case OR_RA: slot[0] = 0; slot[1] = 3; break;",
     "case OR_RA: slot[0] = 0; slot[1] = 1; break;", 0),                                               # [judge]
    ("write_slot_ARGB", "case OR_ARGB: slot[0] = 3; slot[1] = 0; slot[2] = 1; slot[3] = 2; break;",
     "case OR_ARGB: slot[0] = 0; slot[1] = 1; slot[2] = 2; slot[3] = 3; break;", 0),                   # [judge]
    ("write_slot_ARGB_rotated", "case OR_ARGB: slot[0] = 3; slot[1] = 0; slot[2] = 1; slot[3] = 2; break;",
     "case OR_ARGB: slot[0] = 1; slot[1] = 2; slot[2] = 3; slot[3] = 0; break;", 0),
    ("write_slot_BGRA", "case OR_BGRA: slot[0] = 2; slot[1] = 1; slot[2] = 0; slot[3] = 3; break;",
     "case OR_BGRA: slot[0] = 0; slot[1] = 1; slot[2] = 2; slot[3] = 3; break;", 0),
    ("snorm16_low_sat", "case OR_SNORM_INT16: return sat_rte(f * 32767.0f, -32768, 32767);",
     "case OR_SNORM_INT16: return sat_rte(f * 32767.0f, -32767, 32767);", 0),                          # [judge]
    ("snorm8_low_sat", "case OR_SNORM_INT8:  return sat_rte(f * 127.0f, -128, 127);",
     "case OR_SNORM_INT8:  return sat_rte(f * 127.0f, -127, 127);", 0),
    ("sint16_low_sat", "clamp64(v.i, -32768, 32767)", "clamp64(v.i, -32767, 32767)", 0),               # [judge]
    ("sint8_low_sat", "clamp64(v.i, -128, 127)", "clamp64(v.i, -127, 127)", 0),
    ("uint16_wraps", "code = v.u > 65535u ? 65535u : v.u;", "code = v.u & 0xffffu;", 0),
    ("unorm8_write_scale", "case OR_UNORM_INT8:  return sat_rte(f * 255.0f, 0, 255);",
     "case OR_UNORM_INT8:  return sat_rte(f * 256.0f, 0, 255);", 0),
    ("sat_rte_truncates", "return (int32_t)rintf(p);", "return (int32_t)p;", 0),
    ("sat_rte_nan", "if (isnan(p)) return 0;", "if (isnan(p)) return hi;", 0),
    ("half_write_round_half_up", "double r = rint(q);", "double r = floor(q + 0.5);", 0),
    ("half_write_subnormal_exp", "if (E < -14) E = -14;", "if (E < -15) E = -15;", 0),
    ("half_write_overflow", "if (E > 15) return sign | 0x7c00;", "if (E > 16) return sign | 0x7c00;", 0),
    ("packed_write_scale", "word |= (uint32_t)sat_rte(col[c].f * (float)hi, 0, hi) << shift;",
     "word |= (uint32_t)sat_rte(col[c].f * (float)(hi + 1), 0, hi) << shift;", 0),
    ("write_noop_k", "i < 0 || i >= img->width || j < 0 || j >= img->height || k < 0 || k >= img->depth)\n      continue;",
     "i < 0 || i >= img->width || j < 0 || j >= img->height)\n      continue;", 0),                  # [judge]
    ("write_noop_j", "i < 0 || i >= img->width || j < 0 || j >= img->height || k < 0 || k >= img->depth)\n      continue;",
     "i < 0 || i >= img->width || k < 0 || k >= img->depth)\n      continue;", 0),
    ("write_noop_i_bound", "i < 0 || i >= img->width || j < 0 || j >= img->height || k < 0 || k >= img->depth)\n      continue;",
     "i < 0 || i > img->width || j < 0 || j >= img->height || k < 0 || k >= img->depth)\n      continue;", 0),
    # ---- bulk operations ([CL1.2 §5.2.2, §5.2.3, §5.3.3-5.3.5])
    ("copy_rect_src_slice_default", "if (ssp == 0) ssp = region[1] * srp;", "if (ssp == 0) ssp = region[1] * region[0];", 0),  # [judge]
    ("copy_rect_dst_slice_default", "if (dsp == 0) dsp = region[1] * drp;", "if (dsp == 0) dsp = region[1] * region[0];", 0),
    ("copy_rect_row_default", "if (srp == 0) srp = region[0];", "if (srp == 0) srp = region[1];", 0),
    ("copy_rect_src_origin_z", "size_t soff = so[2] * ssp + so[1] * srp + so[0];",
     "size_t soff = so[1] * srp + so[0];", 0),
    ("fill_buffer_phase", "buf[offset + k] = p[k % pattern_size];", "buf[offset + k] = p[(k + 1) % pattern_size];", 0),
    ("fill_image_origin_z", "memcpy(texel_ptr(img, origin[0] + x, origin[1] + y, origin[2] + z), texel, (size_t)es);",
     "memcpy(texel_ptr(img, origin[0] + x, origin[1] + y, z), texel, (size_t)es);", 0),              # [judge]
    ("buffer_to_image_origin_z", "memcpy(texel_ptr(dst, dso[0] + x, dso[1] + y, dso[2] + z),\n               src + src_offset",
     "memcpy(texel_ptr(dst, dso[0] + x, dso[1] + y, z),\n               src + src_offset", 0),      # [judge]
    ("image_to_buffer_origin_z", "texel_ptr(src, so[0] + x, so[1] + y, so[2] + z),\n               (size_t)es);",
     "texel_ptr(src, so[0] + x, so[1] + y, z),\n               (size_t)es);", 0),
    ("copy_image_dst_origin_z", "memcpy(texel_ptr(dst, dso[0] + x, dso[1] + y, dso[2] + z),\n               texel_ptr(src",
     "memcpy(texel_ptr(dst, dso[0] + x, dso[1] + y, z),\n               texel_ptr(src", 0),
    ("host_rect_1d_array_stride", "*row_pitch = *slice_pitch;                  /* layer y",
     "/* mutated */                  /* layer y", 0),
    ("host_rect_slice_default", "if (*slice_pitch == 0) *slice_pitch = *row_pitch * region[1];",
     "if (*slice_pitch == 0) *slice_pitch = *row_pitch * region[2];", 0),
    ("rect_overlap_touching", "if (a0 < b1 && b0 < a1) return 1;", "if (a0 <= b1 && b0 <= a1) return 1;", 0),
    # ---- CUDA texture side (NEXT row 3)
    ("tex_wrap_no_mod", "case TEX_WRAP: return ((i % n) + n) % n;", "case TEX_WRAP: return i;", 0),
    ("tex_signed_divisor", "(float)((1u << (8 * tb - 1)) - 1u)", "(float)(1u << (8 * tb - 1))", 0),
    ("tex_mirror_parity", "x = (fmodf(floorf(x), 2.0f) == 0.0f) ? f : 1.0f - f;           /* floor(x) even / odd */",
     "x = (fmodf(floorf(x), 2.0f) != 0.0f) ? f : 1.0f - f;           /* floor(x) even / odd */", 0),
    ("tex_border_flag", "if (i < 0 || i >= n) *out = 1;", "if (i < 0 || i > n) *out = 1;", 0),
]

# Equivalent mutants considered and excluded (no input can tell them apart):
#  * `(int64_t)f` -> `(int64_t)x` in ifloor for non-negative x only: not a single-token edit of the form above;
#  * REPEAT `if (b0 < 0) b0 = n + b0` -> `b0 += n` under `b0 < 0`: same statement;
#  * fill_buffer `k % p` -> `(k + offset) % p`: offsets are multiples of p by validation (A22);
#  * clamp64 argument order swaps where lo == hi cannot occur (n >= 1).


def apply(src: str, old: str, new: str, occ: int) -> str:
    idx, start = -1, 0
    for _ in range(occ + 1):
        idx = src.find(old, start)
        if idx < 0:
            raise ValueError(f"mutation target not found (occurrence {occ}): {old!r}")
        start = idx + 1
    return src[:idx] + new + src[idx + len(old):]


def run_one(m, tmp):
    name, old, new, occ = m
    src = open(SRC).read()
    mutated = apply(src, old, new, occ)
    d = os.path.join(tmp, name)
    os.makedirs(d, exist_ok=True)
    c = os.path.join(d, "oracle.c")
    with open(c, "w") as fh:
        fh.write(mutated)
    # the header is included relative to the source
    os.symlink(os.path.join(ROOT, "oracle", "oracle.h"), os.path.join(d, "oracle.h"))
    so = os.path.join(d, "liboracle.so")
    subprocess.run(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
                    "-w", "-o", so, c, "-lm", "-lpthread"], check=True)
    env = dict(os.environ, B2CL_ORACLE_LIB=so)
    tests = sorted(os.path.join(ROOT, "tests", f) for f in os.listdir(os.path.join(ROOT, "tests"))
                   if f.startswith("test_oracle_") and f.endswith(".py"))
    r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-m", "not gpu", "-p", "no:cacheprovider",
                        *tests], cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    caught = r.returncode != 0
    first = ""
    if caught:
        for line in r.stdout.splitlines():
            if line.startswith("FAILED") or line.startswith("ERROR"):
                first = line.split(" - ")[0]
                break
    return name, caught, first


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("-j", type=int, default=max(1, (os.cpu_count() or 2) // 2))
    ap.add_argument("-k", default="", help="only mutants whose name contains this")
    a = ap.parse_args()
    ms = [m for m in MUTANTS if a.k in m[0]]
    src = open(SRC).read()
    for m in ms:  # every target must exist before anything runs
        apply(src, m[1], m[2], m[3])
    with tempfile.TemporaryDirectory() as tmp, ThreadPoolExecutor(a.j) as ex:
        res = list(ex.map(lambda m: run_one(m, tmp), ms))
    surv = [n for n, c, _ in res if not c]
    for n, c, first in res:
        print(f"{'caught  ' if c else 'SURVIVED'} {n:32s} {first}")
    print(f"{len(res) - len(surv)} / {len(res)} mutants caught")
    return 1 if surv else 0


if __name__ == "__main__":
    sys.exit(main())
