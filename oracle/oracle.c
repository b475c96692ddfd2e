/*
 * oracle.c -- plain, slow, CPU oracle of the OpenCL 1.2 image / sampler /
 * memory-object rules emulated by the b2cl hot path.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h).  Nothing in the product path
 * includes, links or calls this file.
 *
 * Compile: gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math (no FMA
 * contraction: SURVEY.md §7 "FP determinism of the address math", reading A2).
 *
 * Citations: P:<n> = /root/reference/PAPER.md line n.  [CL1.2 §x] = the
 * Khronos OpenCL 1.2 specification, which the paper names as its target
 * and to which it delegates all image semantics ("We support all
 * OpenCL image-related functions").  A<n> = the reading taken where
 * the spec is silent (restated in DESIGN.md §3).
 */
#define _GNU_SOURCE
#include "oracle.h"

#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------ */
/* Formats: channel order and channel data type ([CL1.2 §5.3.1.1])      */
/* ------------------------------------------------------------------ */

static int type_bytes(uint32_t type) {
  switch (type) {
    case OR_SNORM_INT8: case OR_UNORM_INT8: case OR_SIGNED_INT8: case OR_UNSIGNED_INT8:
      return 1;
    case OR_SNORM_INT16: case OR_UNORM_INT16: case OR_SIGNED_INT16:
    case OR_UNSIGNED_INT16: case OR_HALF_FLOAT:
      return 2;
    case OR_SIGNED_INT32: case OR_UNSIGNED_INT32: case OR_FLOAT:
      return 4;
    default:
      return -1;
  }
}

/* The packed channel types ([CL1.2 §5.3.1.1]): a normalized 5-6-5 RGB, or
 * x-5-5-5 / x-10-10-10 xRGB, in one 16- or 32-bit little-endian word, legal
 * only with the orders CL_RGB and CL_RGBx. */
static int is_packed(uint32_t type) {
  return type == OR_UNORM_SHORT_565 || type == OR_UNORM_SHORT_555 || type == OR_UNORM_INT_101010;
}

/* width and lowest bit of stored channel c (0 = R, 1 = G, 2 = B) of a packed word */
static void packed_field(uint32_t type, int c, int* bits, int* shift) {
  static const int w565[3] = {5, 6, 5}, s565[3] = {11, 5, 0};
  static const int w555[3] = {5, 5, 5}, s555[3] = {10, 5, 0};
  static const int w10[3] = {10, 10, 10}, s10[3] = {20, 10, 0};
  const int *w = w10, *sh = s10;
  if (type == OR_UNORM_SHORT_565) { w = w565; sh = s565; }
  if (type == OR_UNORM_SHORT_555) { w = w555; sh = s555; }
  *bits = w[c];
  *shift = sh[c];
}

int oracle_channels(uint32_t order) {
  switch (order) {
    case OR_R: case OR_A: case OR_INTENSITY: case OR_LUMINANCE: return 1;
    case OR_RG: case OR_RA: return 2;
    case OR_RGB: case OR_RGBx: return 3;   /* packed types only */
    case OR_RGBA: case OR_BGRA: case OR_ARGB: return 4;
    default: return -1; /* CL_Rx, CL_RGx: not supported (reading A37) */
  }
}

/* The [CL1.2 §5.3.1.1] table of legal (order, type) pairs. */
static int format_ok(uint32_t order, uint32_t type) {
  if (oracle_channels(order) < 0) return 0;
  /* "CL_RGB or CL_RGBx: only if the channel data type is CL_UNORM_SHORT_565,
     CL_UNORM_SHORT_555 or CL_UNORM_INT_101010" -- and those types need them */
  if (order == OR_RGB || order == OR_RGBx || is_packed(type))
    return (order == OR_RGB || order == OR_RGBx) && is_packed(type);
  if (type_bytes(type) < 0) return 0;
  if (order == OR_BGRA || order == OR_ARGB)
    return type == OR_UNORM_INT8 || type == OR_SNORM_INT8 || type == OR_SIGNED_INT8 ||
           type == OR_UNSIGNED_INT8;
  if (order == OR_INTENSITY || order == OR_LUMINANCE)
    return type == OR_UNORM_INT8 || type == OR_UNORM_INT16 || type == OR_SNORM_INT8 ||
           type == OR_SNORM_INT16 || type == OR_HALF_FLOAT || type == OR_FLOAT;
  return 1;
}

int oracle_elem_size(uint32_t order, uint32_t type) {
  if (!format_ok(order, type)) return -1;
  if (is_packed(type)) return type == OR_UNORM_INT_101010 ? 4 : 2;  /* one packed word */
  return oracle_channels(order) * type_bytes(type); /* elem_size, Fig. 6 */
}

/* read_imagef applies to normalized-int, half and float types; read_imagei to
 * SIGNED_INT*; read_imageui to UNSIGNED_INT* ([CL1.2 §6.12.14.2]).  Any other
 * pairing is undefined in the spec and rejected here (reading A7). */
static int rtype_of(uint32_t type) {
  switch (type) {
    case OR_SIGNED_INT8: case OR_SIGNED_INT16: case OR_SIGNED_INT32: return OR_RT_I;
    case OR_UNSIGNED_INT8: case OR_UNSIGNED_INT16: case OR_UNSIGNED_INT32: return OR_RT_UI;
    default: return OR_RT_F;
  }
}

/* ------------------------------------------------------------------ */
/* Half precision, written out from the IEEE 754 binary16 definition    */
/* ------------------------------------------------------------------ */

float oracle_half_to_float(uint16_t h) {
  int sign = (h >> 15) & 1;
  int e = (h >> 10) & 31;
  int m = h & 1023;
  double v;
  if (e == 0) {
    v = ldexp((double)m, -24);              /* subnormal: m * 2^-24 */
  } else if (e == 31) {
    if (m == 0) v = INFINITY;
    else return sign ? -NAN : NAN;
  } else {
    v = ldexp((double)(1024 + m), e - 25);  /* (1 + m/1024) * 2^(e-15) */
  }
  return (float)(sign ? -v : v);            /* exact: every half is a float */
}

/* Round-to-nearest-even float -> half, keeping subnormals; overflow -> inf;
 * NaN -> quiet NaN (reading A13, [CL1.2 §8.3.2]). */
uint16_t oracle_float_to_half_rte(float f) {
  uint16_t sign = signbit(f) ? 0x8000 : 0;
  double v = fabs((double)f);
  if (isnan(f)) return sign | 0x7e00;
  if (v == 0.0) return sign;
  if (isinf(f)) return sign | 0x7c00;
  int e;
  frexp(v, &e);                   /* v = m * 2^e, m in [0.5, 1) */
  int E = e - 1;                  /* unbiased exponent of v */
  if (E < -14) E = -14;           /* subnormal range: fixed quantum 2^-24 */
  double q = ldexp(v, 10 - E);    /* significand scaled to 10 fraction bits */
  double r = rint(q);             /* half-even (default rounding mode), exact input */
  if (r >= 2048.0) { r = r / 2.0; E += 1; }
  if (E > 15) return sign | 0x7c00;
  if (r < 1024.0) return sign | (uint16_t)r;            /* subnormal (E == -14) */
  return sign | (uint16_t)(((E + 15) << 10) | ((int)r - 1024));
}

/* ------------------------------------------------------------------ */
/* Normalized integer conversions ([CL1.2 §8.3.1], readings A11, A12)   */
/* ------------------------------------------------------------------ */

float oracle_norm_to_float(uint32_t type, int32_t code) {
  switch (type) {
    case OR_UNORM_INT8:  return (float)code / 255.0f;
    case OR_UNORM_INT16: return (float)code / 65535.0f;
    case OR_SNORM_INT8:  return fmaxf(-1.0f, (float)code / 127.0f);
    case OR_SNORM_INT16: return fmaxf(-1.0f, (float)code / 32767.0f);
    default: return NAN;
  }
}

/* convert_<T>_sat_rte(f * scale): the product is one fp32 RN multiply, then
 * round half to even, saturate; NaN -> 0 (reading A12). */
static int32_t sat_rte(float p, int32_t lo, int32_t hi) {
  if (isnan(p)) return 0;
  if (p <= (float)lo) return lo;
  if (p >= (float)hi) return hi;
  return (int32_t)rintf(p);
}

int32_t oracle_float_to_norm(uint32_t type, float f) {
  switch (type) {
    case OR_UNORM_INT8:  return sat_rte(f * 255.0f, 0, 255);
    case OR_UNORM_INT16: return sat_rte(f * 65535.0f, 0, 65535);
    case OR_SNORM_INT8:  return sat_rte(f * 127.0f, -128, 127);
    case OR_SNORM_INT16: return sat_rte(f * 32767.0f, -32768, 32767);
    default: return 0;
  }
}

/* ------------------------------------------------------------------ */
/* Texel fetch and channel mapping ([CL1.2 §8.3], table in §6.12.14.1)  */
/* ------------------------------------------------------------------ */

/* One stored channel code as a little-endian integer of the channel width. */
static int64_t load_code(const uint8_t* p, uint32_t type) {
  switch (type) {
    case OR_SNORM_INT8: case OR_SIGNED_INT8: return (int8_t)p[0];
    case OR_UNORM_INT8: case OR_UNSIGNED_INT8: return p[0];
    case OR_SNORM_INT16: case OR_SIGNED_INT16: {
      int16_t v; memcpy(&v, p, 2); return v;
    }
    case OR_UNORM_INT16: case OR_UNSIGNED_INT16: case OR_HALF_FLOAT: {
      uint16_t v; memcpy(&v, p, 2); return v;
    }
    case OR_SIGNED_INT32: { int32_t v; memcpy(&v, p, 4); return v; }
    case OR_UNSIGNED_INT32: case OR_FLOAT: { uint32_t v; memcpy(&v, p, 4); return v; }
    default: return 0;
  }
}

/* Memory channel slots -> (x,y,z,w).  mem[] holds the channels in the order
 * they are stored (BGRA = B,G,R,A; ARGB = A,R,G,B).  zero/one are the
 * defaults for missing components (0.0/1.0 or 0/1). */
typedef union { float f; uint32_t u; int32_t i; } val32;

static void map_to_xyzw(uint32_t order, const val32* mem, val32 zero, val32 one, val32* out) {
  switch (order) {
    case OR_R:         out[0] = mem[0]; out[1] = zero;   out[2] = zero;   out[3] = one;    break;
    case OR_A:         out[0] = zero;   out[1] = zero;   out[2] = zero;   out[3] = mem[0]; break;
    case OR_RG:        out[0] = mem[0]; out[1] = mem[1]; out[2] = zero;   out[3] = one;    break;
    case OR_RA:        out[0] = mem[0]; out[1] = zero;   out[2] = zero;   out[3] = mem[1]; break;
    case OR_RGBA:      out[0] = mem[0]; out[1] = mem[1]; out[2] = mem[2]; out[3] = mem[3]; break;
    case OR_BGRA:      out[0] = mem[2]; out[1] = mem[1]; out[2] = mem[0]; out[3] = mem[3]; break;
    case OR_ARGB:      out[0] = mem[1]; out[1] = mem[2]; out[2] = mem[3]; out[3] = mem[0]; break;
    case OR_INTENSITY: out[0] = mem[0]; out[1] = mem[0]; out[2] = mem[0]; out[3] = mem[0]; break;
    case OR_LUMINANCE: out[0] = mem[0]; out[1] = mem[0]; out[2] = mem[0]; out[3] = one;    break;
    case OR_RGB:       out[0] = mem[0]; out[1] = mem[1]; out[2] = mem[2]; out[3] = one;    break;
    case OR_RGBx:      out[0] = mem[0]; out[1] = mem[1]; out[2] = mem[2]; out[3] = one;    break;
    default:           out[0] = zero;   out[1] = zero;   out[2] = zero;   out[3] = zero;   break;
  }
}

/* Border colour of CLK_ADDRESS_CLAMP ([CL1.2 §6.12.14.1]; reading A4 extends
 * it to CLK_ADDRESS_NONE out of range): (0,0,0,0) for A, INTENSITY, Rx, RA,
 * RGx, RGBx, ARGB, BGRA, RGBA; (0,0,0,1) for R, RG, RGB, LUMINANCE.  (So for
 * CL_RGBx the border's alpha 0 differs from an in-range texel's alpha 1.) */
static void border_color(uint32_t order, val32 zero, val32 one, val32* out) {
  out[0] = zero; out[1] = zero; out[2] = zero;
  out[3] = (order == OR_R || order == OR_RG || order == OR_RGB || order == OR_LUMINANCE)
               ? one : zero;
}

/* Read texel (i,j,k) converted for return class rtype; border if out of range. */
static void fetch(const oracle_image* img, int64_t i, int64_t j, int64_t k, int rtype,
                  val32* out) {
  val32 zero, one;
  if (rtype == OR_RT_F) { zero.f = 0.0f; one.f = 1.0f; }
  else { zero.u = 0; one.u = 1; }
  if (i < 0 || i >= img->width || j < 0 || j >= img->height || k < 0 || k >= img->depth) {
    border_color(img->order, zero, one, out);
    return;
  }
  int nc = oracle_channels(img->order);
  int tb = type_bytes(img->type);
  int es = oracle_elem_size(img->order, img->type);
  const uint8_t* p = img->data + k * img->slice_pitch + j * img->row_pitch +
                     i * (int64_t)es;
  val32 mem[4];
  if (is_packed(img->type)) {
    /* the word, little endian; each field c / (2^bits - 1) ([CL1.2 §8.3.1.1],
       correctly rounded as for the other normalized types, reading A11) */
    uint32_t word = 0;
    for (int b = 0; b < es; ++b) word |= (uint32_t)p[b] << (8 * b);
    for (int c = 0; c < 3; ++c) {
      int bits, shift;
      packed_field(img->type, c, &bits, &shift);
      uint32_t code = (word >> shift) & ((1u << bits) - 1u);
      mem[c].f = (float)code / (float)((1u << bits) - 1u);
    }
    map_to_xyzw(img->order, mem, zero, one, out);
    return;
  }
  for (int c = 0; c < nc; ++c) {
    int64_t code = load_code(p + c * tb, img->type);
    switch (img->type) {
      case OR_UNORM_INT8: case OR_UNORM_INT16: case OR_SNORM_INT8: case OR_SNORM_INT16:
        mem[c].f = oracle_norm_to_float(img->type, (int32_t)code); break;
      case OR_HALF_FLOAT: mem[c].f = oracle_half_to_float((uint16_t)code); break;
      case OR_FLOAT: mem[c].u = (uint32_t)code; break;       /* bit copy (A14) */
      default: mem[c].i = (int32_t)code; break;               /* sign/zero-extended */
    }
  }
  map_to_xyzw(img->order, mem, zero, one, out);
}

/* ------------------------------------------------------------------ */
/* Addressing ([CL1.2 §8.2]; readings A2, A3)                          */
/* ------------------------------------------------------------------ */

/* (int)floor(x), saturating to int32 with NaN -> 0 (reading A3). */
static int64_t ifloor(float x) {
  if (isnan(x)) return 0;
  float f = floorf(x);
  if (f >= 2147483648.0f) return INT32_MAX;
  if (f < -2147483648.0f) return INT32_MIN;
  return (int64_t)f;
}

static int64_t clamp64(int64_t v, int64_t lo, int64_t hi) {
  return v < lo ? lo : (v > hi ? hi : v);
}

/* address_mode() of the non-wrapping modes. */
static int64_t am(uint32_t addressing, int64_t i, int64_t n) {
  switch (addressing) {
    case OR_ADDRESS_CLAMP_TO_EDGE: return clamp64(i, 0, n - 1);
    case OR_ADDRESS_CLAMP:         return clamp64(i, -1, n);
    default:                       return i;            /* CLK_ADDRESS_NONE */
  }
}

void oracle_axis_nearest(float s, int64_t n, int normalized, uint32_t addressing,
                         int64_t* i0) {
  float fn = (float)n;
  if (addressing == OR_ADDRESS_REPEAT) {
    /* u = (s - floor(s)) * wt; i = (int)floor(u); if (i > wt - 1) i = i - wt */
    float u = (s - floorf(s)) * fn;
    int64_t i = ifloor(u);
    if (i > n - 1) i = i - n;
    *i0 = i;
  } else if (addressing == OR_ADDRESS_MIRRORED_REPEAT) {
    /* s' = 2.0f*rint(0.5f*s); s' = fabs(s - s'); u = s'*wt; i = min((int)floor(u), wt-1) */
    float sp = 2.0f * rintf(0.5f * s);
    sp = fabsf(s - sp);
    float u = sp * fn;
    int64_t i = ifloor(u);
    *i0 = i < n - 1 ? i : n - 1;
  } else {
    /* u = normalized ? s * wt : s; i = address_mode((int)floor(u)) */
    float u = normalized ? s * fn : s;
    *i0 = am(addressing, ifloor(u), n);
  }
}

void oracle_axis_linear(float s, int64_t n, int normalized, uint32_t addressing,
                        int64_t* i0, int64_t* i1, float* a) {
  float fn = (float)n;
  if (addressing == OR_ADDRESS_REPEAT) {
    /* u = (s - floor(s))*wt; i0 = (int)floor(u - 0.5); i1 = i0 + 1;
       if (i0 < 0) i0 = wt + i0; if (i1 > wt - 1) i1 = i1 - wt; a = frac(u - 0.5) */
    float u = (s - floorf(s)) * fn;
    float t = u - 0.5f;
    int64_t b0 = ifloor(t);
    int64_t b1 = b0 + 1;
    if (b0 < 0) b0 = n + b0;
    if (b1 > n - 1) b1 = b1 - n;
    *i0 = b0; *i1 = b1;
    *a = t - floorf(t);
  } else if (addressing == OR_ADDRESS_MIRRORED_REPEAT) {
    /* s' as for NEAREST; u = s'*wt; i0 = (int)floor(u - 0.5); i1 = i0 + 1;
       i0 = max(i0, 0); i1 = min(i1, wt - 1); a = frac(u - 0.5) */
    float sp = 2.0f * rintf(0.5f * s);
    sp = fabsf(s - sp);
    float u = sp * fn;
    float t = u - 0.5f;
    int64_t b0 = ifloor(t);
    int64_t b1 = b0 + 1;
    *i0 = b0 > 0 ? b0 : 0;
    *i1 = b1 < n - 1 ? b1 : n - 1;
    *a = t - floorf(t);
  } else {
    /* i0 = address_mode((int)floor(u - 0.5)); i1 = address_mode((int)floor(u - 0.5) + 1);
       a = frac(u - 0.5) */
    float u = normalized ? s * fn : s;
    float t = u - 0.5f;
    int64_t b = ifloor(t);
    *i0 = am(addressing, b, n);
    *i1 = am(addressing, b + 1, n);      /* +1 in int64: no overflow (A3) */
    *a = t - floorf(t);
  }
}

/* ------------------------------------------------------------------ */
/* read_imagef / read_imagei / read_imageui                             */
/* ------------------------------------------------------------------ */

static int check_read(const oracle_image* img, int normalized, uint32_t addressing,
                      uint32_t filter, int rtype) {
  if (oracle_elem_size(img->order, img->type) < 0) return OR_IMAGE_FORMAT_NOT_SUPPORTED;
  if (addressing < OR_ADDRESS_NONE || addressing > OR_ADDRESS_MIRRORED_REPEAT) return OR_INVALID_VALUE;
  if (filter != OR_FILTER_NEAREST && filter != OR_FILTER_LINEAR) return OR_INVALID_VALUE;
  if (!normalized && (addressing == OR_ADDRESS_REPEAT || addressing == OR_ADDRESS_MIRRORED_REPEAT))
    return OR_INVALID_VALUE;                                  /* A5 */
  if (rtype != rtype_of(img->type)) return OR_INVALID_OPERATION;   /* A7 */
  if (rtype != OR_RT_F && filter == OR_FILTER_LINEAR) return OR_INVALID_OPERATION; /* A6 */
  return OR_SUCCESS;
}

static void store16(const val32* v, void* out16) { memcpy(out16, v, 16); }

/* [CL1.2 §8.4] "Selecting an Image from an Image Array": the layer is
 * clamp(rint(w), 0, d - 1); rintf rounds half to even in the default mode. */
int64_t oracle_layer_index(float c, int64_t n) {
  if (isnan(c)) return 0;                                    /* A35 */
  float r = rintf(c);
  int64_t l = r >= 2147483648.0f ? INT32_MAX : (r < -2147483648.0f ? INT32_MIN : (int64_t)r);
  return clamp64(l, 0, n - 1);
}

static void sample_checked(const oracle_image* img, int normalized, uint32_t addressing,
                           uint32_t filter, int rtype, const float* coord, void* out16) {
  int dims = img->dims, nc = dims + (img->arrayed ? 1 : 0);
  int64_t n[3] = {img->width, img->height, img->depth};
  float c[3] = {coord[0], nc > 1 ? coord[1] : 0.0f, nc > 2 ? coord[2] : 0.0f};
  /* an array's layer axis (the one after the sampled axes) is selected, not
     addressed: the sampler's normalization, addressing and filter skip it */
  int64_t layer = img->arrayed ? oracle_layer_index(c[dims], n[dims]) : 0;
  if (filter == OR_FILTER_NEAREST) {
    int64_t ix[3] = {0, 0, 0};
    for (int d = 0; d < dims; ++d) oracle_axis_nearest(c[d], n[d], normalized, addressing, &ix[d]);
    if (img->arrayed) ix[dims] = layer;
    val32 t[4];
    fetch(img, ix[0], ix[1], ix[2], rtype, t);
    store16(t, out16);
    return;
  }
  /* LINEAR: T = sum over taps of the weight products times the texel
     ([CL1.2 §8.2] 1D/2D/3D formulas), evaluated in fp64, rounded once (O6). */
  int64_t lo[3] = {0, 0, 0}, hi[3] = {0, 0, 0};
  float w[3] = {0.0f, 0.0f, 0.0f};
  for (int d = 0; d < dims; ++d)
    oracle_axis_linear(c[d], n[d], normalized, addressing, &lo[d], &hi[d], &w[d]);
  if (img->arrayed) lo[dims] = hi[dims] = layer;   /* one layer, weight 1 */
  double acc[4] = {0.0, 0.0, 0.0, 0.0};
  int nk = dims > 2 ? 2 : 1, nj = dims > 1 ? 2 : 1;
  for (int kk = 0; kk < nk; ++kk) {
    double wk = dims > 2 ? (kk ? (double)w[2] : 1.0 - (double)w[2]) : 1.0;
    for (int jj = 0; jj < nj; ++jj) {
      double wj = dims > 1 ? (jj ? (double)w[1] : 1.0 - (double)w[1]) : 1.0;
      for (int ii = 0; ii < 2; ++ii) {
        double wi = ii ? (double)w[0] : 1.0 - (double)w[0];
        val32 t[4];
        fetch(img, ii ? hi[0] : lo[0], jj ? hi[1] : lo[1], kk ? hi[2] : lo[2], OR_RT_F, t);
        double wt = wi * wj * wk;
        for (int ch = 0; ch < 4; ++ch) acc[ch] += wt * (double)t[ch].f;
      }
    }
  }
  val32 r[4];
  for (int ch = 0; ch < 4; ++ch) r[ch].f = (float)acc[ch];
  store16(r, out16);
}

int oracle_read_image(const oracle_image* img, int normalized, uint32_t addressing,
                      uint32_t filter, int rtype, const float* coord, void* out16) {
  int st = check_read(img, normalized, addressing, filter, rtype);
  if (st != OR_SUCCESS) return st;
  sample_checked(img, normalized, addressing, filter, rtype, coord, out16);
  return OR_SUCCESS;
}

/* Integer coordinates (reading A30): legal only with unnormalized coordinates,
 * NEAREST and a non-wrapping mode.  The coordinate is the texel index itself,
 * i = address_mode(coord) ([CL1.2 §8.2] with floor(u) = coord exactly), and an
 * array's layer is clamp(coord, 0, n - 1) ([CL1.2 §8.4]: rint of an integer
 * is itself).  For |coord| <= 2^24 this is the float path at u = (float)coord;
 * beyond, it stays exact (1D image buffers reach 2^31 - 1 texels). */
int oracle_read_image_icoord(const oracle_image* img, int normalized, uint32_t addressing,
                             uint32_t filter, int rtype, const int32_t* icoord, void* out16) {
  int st = check_read(img, normalized, addressing, filter, rtype);
  if (st != OR_SUCCESS) return st;
  if (normalized || filter != OR_FILTER_NEAREST || addressing == OR_ADDRESS_REPEAT ||
      addressing == OR_ADDRESS_MIRRORED_REPEAT)
    return OR_INVALID_OPERATION;
  int64_t n[3] = {img->width, img->height, img->depth};
  int64_t ix[3] = {0, 0, 0};
  for (int d = 0; d < img->dims; ++d) ix[d] = am(addressing, icoord[d], n[d]);
  if (img->arrayed) ix[img->dims] = clamp64(icoord[img->dims], 0, n[img->dims] - 1);
  val32 t[4];
  fetch(img, ix[0], ix[1], ix[2], rtype, t);
  store16(t, out16);
  return OR_SUCCESS;
}

int oracle_read_samples(const oracle_image* img, int normalized, uint32_t addressing,
                        uint32_t filter, int rtype, int coord_is_int, const void* coords,
                        int64_t cstride, int64_t n, void* out) {
  for (int64_t s = 0; s < n; ++s) {
    int st;
    if (coord_is_int)
      st = oracle_read_image_icoord(img, normalized, addressing, filter, rtype,
                                    (const int32_t*)coords + s * cstride,
                                    (uint8_t*)out + 16 * s);
    else
      st = oracle_read_image(img, normalized, addressing, filter, rtype,
                             (const float*)coords + s * cstride, (uint8_t*)out + 16 * s);
    if (st != OR_SUCCESS) return st;
  }
  return OR_SUCCESS;
}

/* ---- grid mode ---- */
typedef struct {
  const oracle_image* img;
  int normalized; uint32_t addressing, filter; int rtype;
  const float* A;
  int64_t out_w, out_h;
  int out_channels;
  int64_t z0, z1, y0, y1;
  uint8_t* out;
  int64_t row_begin, row_end;  /* rows of the (z,y) sub-box this worker computes */
} grid_job;

static void grid_rows(const grid_job* g) {
  int64_t ny = g->y1 - g->y0;
  int dims = g->img->dims + (g->img->arrayed ? 1 : 0);   /* + the layer coordinate */
  for (int64_t r = g->row_begin; r < g->row_end; ++r) {
    int64_t z = g->z0 + r / ny, y = g->y0 + r % ny;
    uint8_t* orow = g->out + r * g->out_w * 4 * g->out_channels;
    for (int64_t x = 0; x < g->out_w; ++x) {
      float xf = (float)x, yf = (float)y, zf = (float)z;
      float c[3];
      for (int k = 0; k < dims; ++k) {
        const float* a = g->A + 4 * k;
        float v = a[0] * xf;     /* one RN op each, in this order (A2) */
        v = v + a[1] * yf;
        v = v + a[2] * zf;
        v = v + a[3];
        c[k] = v;
      }
      uint8_t res[16];
      sample_checked(g->img, g->normalized, g->addressing, g->filter, g->rtype, c, res);
      memcpy(orow + x * 4 * g->out_channels, res, 4 * g->out_channels);
    }
  }
}

static void* grid_worker(void* arg) { grid_rows((const grid_job*)arg); return NULL; }

int oracle_read_grid(const oracle_image* img, int normalized, uint32_t addressing,
                     uint32_t filter, int rtype, const float* affine12,
                     int64_t out_w, int64_t out_h, int64_t out_d, int out_channels,
                     int64_t z0, int64_t z1, int64_t y0, int64_t y1,
                     void* out, int nthreads) {
  int st = check_read(img, normalized, addressing, filter, rtype);
  if (st != OR_SUCCESS) return st;
  if (out_channels < 1 || out_channels > 4) return OR_INVALID_VALUE;
  if (z0 < 0 || z1 > out_d || z0 > z1 || y0 < 0 || y1 > out_h || y0 > y1) return OR_INVALID_VALUE;
  int64_t rows = (z1 - z0) * (y1 - y0);
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 256) nthreads = 256;
  if (rows < nthreads) nthreads = rows > 0 ? (int)rows : 1;
  grid_job jobs[256];
  pthread_t tid[256];
  for (int t = 0; t < nthreads; ++t) {
    grid_job g = {img, normalized, addressing, filter, rtype, affine12, out_w, out_h,
                  out_channels, z0, z1, y0, y1, (uint8_t*)out,
                  rows * t / nthreads, rows * (t + 1) / nthreads};
    jobs[t] = g;
  }
  if (nthreads == 1) {
    grid_rows(&jobs[0]);
    return OR_SUCCESS;
  }
  for (int t = 0; t < nthreads; ++t) pthread_create(&tid[t], NULL, grid_worker, &jobs[t]);
  for (int t = 0; t < nthreads; ++t) pthread_join(tid[t], NULL);
  return OR_SUCCESS;
}

/* ------------------------------------------------------------------ */
/* CUDA texture fetches ([CUDA-PG TF]: the CUDA C Programming Guide,     */
/* appendix "Texture Fetching"; the source side of P:449)               */
/* ------------------------------------------------------------------ */

enum { TEX_WRAP = 0, TEX_CLAMP = 1, TEX_MIRROR = 2, TEX_BORDER = 3 };
enum { TEX_POINT = 0, TEX_LINEAR = 1 };
enum { TEX_ELEMENT = 0, TEX_NORMALIZED = 1 };

/* stored channel kind: 0 unsigned int, 1 signed int, 2 floating point */
static int tex_kind(uint32_t type) {
  switch (type) {
    case OR_UNORM_INT8: case OR_UNORM_INT16: case OR_UNSIGNED_INT8: case OR_UNSIGNED_INT16:
    case OR_UNSIGNED_INT32: return 0;
    case OR_SNORM_INT8: case OR_SNORM_INT16: case OR_SIGNED_INT8: case OR_SIGNED_INT16:
    case OR_SIGNED_INT32: return 1;
    default: return 2;
  }
}

/* cudaReadModeNormalizedFloat applies to 8- and 16-bit integer channels. */
static int tex_check(const oracle_image* img, uint32_t read_mode, int filtering_linear) {
  if (img->order != OR_R && img->order != OR_RG && img->order != OR_RGBA)
    return OR_IMAGE_FORMAT_NOT_SUPPORTED;                    /* 1, 2 or 4 channels */
  if (oracle_elem_size(img->order, img->type) < 0) return OR_IMAGE_FORMAT_NOT_SUPPORTED;
  int kind = tex_kind(img->type), tb = type_bytes(img->type);
  if (read_mode == TEX_NORMALIZED && (kind == 2 || tb == 4)) return OR_INVALID_VALUE;
  if (read_mode != TEX_ELEMENT && read_mode != TEX_NORMALIZED) return OR_INVALID_VALUE;
  /* "linear filtering ... only for textures configured to return floating-point data" */
  if (filtering_linear && read_mode == TEX_ELEMENT && kind != 2) return OR_INVALID_OPERATION;
  return OR_SUCCESS;
}

/* Texel (i,j,k) as the fetch returns it; 0 in every component when `zero`. */
static void tex_texel(const oracle_image* img, uint32_t read_mode, int64_t i, int64_t j,
                      int64_t k, int zero, val32* out) {
  for (int c = 0; c < 4; ++c) out[c].u = 0;
  if (zero) return;
  int nc = oracle_channels(img->order), tb = type_bytes(img->type);
  const uint8_t* p = img->data + k * img->slice_pitch + j * img->row_pitch + i * (int64_t)(nc * tb);
  for (int c = 0; c < nc; ++c) {
    int64_t code = load_code(p + c * tb, img->type);
    int kind = tex_kind(img->type);
    if (img->type == OR_FLOAT) {
      out[c].u = (uint32_t)code;
    } else if (img->type == OR_HALF_FLOAT) {
      out[c].f = oracle_half_to_float((uint16_t)code);
    } else if (read_mode == TEX_NORMALIZED) {
      /* unsigned: c / (2^b - 1); signed: c / (2^(b-1) - 1), the most negative
         code clamped to -1.0 (reading A42) */
      float d = kind == 0 ? (float)((1u << (8 * tb)) - 1u) : (float)((1u << (8 * tb - 1)) - 1u);
      float v = (float)code / d;
      out[c].f = v < -1.0f ? -1.0f : v;
    } else {
      out[c].i = (int32_t)code;                              /* element type */
    }
  }
}

/* One axis of a point fetch: the texel index, or *out = 1 for the border. */
static int64_t tex_axis_point(float x, int64_t n, int normalized, uint32_t mode, int* out) {
  float fn = (float)n;
  *out = 0;
  if (normalized) {
    if (mode == TEX_WRAP) x = x - floorf(x);                         /* frac(x) */
    else if (mode == TEX_MIRROR) {
      float f = x - floorf(x);
      x = (fmodf(floorf(x), 2.0f) == 0.0f) ? f : 1.0f - f;           /* floor(x) even / odd */
    }
    x = x * fn;
  }
  int64_t i = ifloor(x);                                              /* i = floor(x) */
  switch (mode) {
    case TEX_WRAP: return ((i % n) + n) % n;   /* frac(x) * N may round to N */
    case TEX_MIRROR: return i < n - 1 ? i : n - 1;
    case TEX_CLAMP: return clamp64(i, 0, n - 1);
    default:
      if (i < 0 || i >= n) *out = 1;                                  /* border */
      return i;
  }
}

/* One axis of a linear fetch: taps i, i+1 of x_B = x - 0.5 and alpha = frac(x_B). */
static void tex_axis_linear(float x, int64_t n, int normalized, uint32_t mode, int64_t* t0,
                            int64_t* t1, int* out0, int* out1, float* alpha) {
  float fn = (float)n;
  if (normalized) {
    if (mode == TEX_WRAP) x = x - floorf(x);
    else if (mode == TEX_MIRROR) {
      float f = x - floorf(x);
      x = (fmodf(floorf(x), 2.0f) == 0.0f) ? f : 1.0f - f;
    }
    x = x * fn;
  }
  float xb = x - 0.5f;                                                /* x_B = x - 0.5 */
  int64_t i = ifloor(xb);                                             /* i = floor(x_B) */
  *alpha = xb - floorf(xb);                                           /* alpha = frac(x_B) */
  int64_t a = i, b = i + 1;
  *out0 = *out1 = 0;
  switch (mode) {
    case TEX_WRAP: a = ((a % n) + n) % n; b = ((b % n) + n) % n; break;
    case TEX_MIRROR:                          /* the mirror repeats the edge texel */
    case TEX_CLAMP: a = clamp64(a, 0, n - 1); b = clamp64(b, 0, n - 1); break;
    default: *out0 = a < 0 || a >= n; *out1 = b < 0 || b >= n; break;
  }
  *t0 = a;
  *t1 = b;
}

int oracle_tex_fetch(const oracle_image* img, const oracle_tex_desc* td, const float* coord,
                     void* out16) {
  int st = tex_check(img, td->read_mode, td->filter_mode == TEX_LINEAR);
  if (st != OR_SUCCESS) return st;
  int dims = img->dims;
  for (int d = 0; d < dims; ++d) {
    uint32_t m = td->address_mode[d];
    if (m > TEX_BORDER) return OR_INVALID_VALUE;
    if (!td->normalized_coords && (m == TEX_WRAP || m == TEX_MIRROR)) return OR_INVALID_VALUE;
  }
  int64_t n[3] = {img->width, img->height, img->depth};
  /* tex1DLayered / tex2DLayered: the integer layer selects the array slice */
  int64_t layer = 0;
  if (img->arrayed) layer = clamp64((int64_t)coord[dims], 0, n[dims] - 1);
  val32 r[4];
  if (td->filter_mode == TEX_POINT) {
    int64_t ix[3] = {0, 0, 0};
    int out = 0;
    for (int d = 0; d < dims; ++d) {
      int o;
      ix[d] = tex_axis_point(coord[d], n[d], td->normalized_coords, td->address_mode[d], &o);
      out |= o;
    }
    if (img->arrayed) ix[dims] = layer;
    tex_texel(img, td->read_mode, ix[0], ix[1], ix[2], out, r);
    memcpy(out16, r, 16);
    return OR_SUCCESS;
  }
  /* tex(x,y,z) = sum over the 2/4/8 taps of the weight products times T,
     evaluated in fp64 and rounded once (reading O6); weights from the fp32
     alpha, beta, gamma (reading A41: not the 8-bit fixed point of the
     texture unit) */
  int64_t lo[3] = {0, 0, 0}, hi[3] = {0, 0, 0};
  int olo[3] = {0, 0, 0}, ohi[3] = {0, 0, 0};
  float w[3] = {0.0f, 0.0f, 0.0f};
  for (int d = 0; d < dims; ++d)
    tex_axis_linear(coord[d], n[d], td->normalized_coords, td->address_mode[d], &lo[d], &hi[d],
                    &olo[d], &ohi[d], &w[d]);
  if (img->arrayed) lo[dims] = hi[dims] = layer;
  double acc[4] = {0.0, 0.0, 0.0, 0.0};
  int nk = dims > 2 ? 2 : 1, nj = dims > 1 ? 2 : 1;
  for (int kk = 0; kk < nk; ++kk) {
    double wk = dims > 2 ? (kk ? (double)w[2] : 1.0 - (double)w[2]) : 1.0;
    for (int jj = 0; jj < nj; ++jj) {
      double wj = dims > 1 ? (jj ? (double)w[1] : 1.0 - (double)w[1]) : 1.0;
      for (int ii = 0; ii < 2; ++ii) {
        double wi = ii ? (double)w[0] : 1.0 - (double)w[0];
        int out = (ii ? ohi[0] : olo[0]) | (jj ? ohi[1] : olo[1]) | (kk ? ohi[2] : olo[2]);
        val32 t[4];
        tex_texel(img, td->read_mode, ii ? hi[0] : lo[0], jj ? hi[1] : lo[1], kk ? hi[2] : lo[2],
                  out, t);
        for (int ch = 0; ch < 4; ++ch) acc[ch] += wi * wj * wk * (double)t[ch].f;
      }
    }
  }
  int nc = oracle_channels(img->order);
  for (int ch = 0; ch < 4; ++ch) r[ch].f = ch < nc ? (float)acc[ch] : 0.0f;
  memcpy(out16, r, 16);
  return OR_SUCCESS;
}

int oracle_tex1Dfetch(const oracle_image* img, uint32_t read_mode, int32_t x, void* out16) {
  int st = tex_check(img, read_mode, 0);
  if (st != OR_SUCCESS) return st;
  val32 r[4];
  tex_texel(img, read_mode, x, 0, 0, x < 0 || x >= img->width, r);
  memcpy(out16, r, 16);
  return OR_SUCCESS;
}

/* ------------------------------------------------------------------ */
/* write_imagef / write_imagei / write_imageui ([CL1.2 §6.12.14.4])     */
/* ------------------------------------------------------------------ */

static void store_code(uint8_t* p, uint32_t type, uint32_t code) {
  int tb = type_bytes(type);
  for (int b = 0; b < tb; ++b) p[b] = (uint8_t)(code >> (8 * b));  /* little endian */
}

int oracle_convert_texel(uint32_t order, uint32_t type, int rtype, const void* color16,
                         uint8_t* texel_out) {
  if (oracle_elem_size(order, type) < 0) return OR_IMAGE_FORMAT_NOT_SUPPORTED;
  if (rtype != rtype_of(type)) return OR_INVALID_OPERATION;   /* A7 */
  val32 col[4];
  memcpy(col, color16, 16);
  /* inverse channel map: which of (x,y,z,w) lands in each memory slot;
     INTENSITY / LUMINANCE store x (reading A16). */
  int slot[4] = {0, 1, 2, 3};
  switch (order) {
    case OR_A: slot[0] = 3; break;
    case OR_RA: slot[0] = 0; slot[1] = 3; break;
    case OR_BGRA: slot[0] = 2; slot[1] = 1; slot[2] = 0; slot[3] = 3; break;
    case OR_ARGB: slot[0] = 3; slot[1] = 0; slot[2] = 1; slot[3] = 2; break;
    default: break;
  }
  if (is_packed(type)) {
    /* R, G, B = convert_sat_rte(x, y, z times 2^bits - 1), the product one fp32
       RN op (reading A12); the unused x bits are written 0 (reading A38) */
    uint32_t word = 0;
    for (int c = 0; c < 3; ++c) {
      int bits, shift;
      packed_field(type, c, &bits, &shift);
      int32_t hi = (int32_t)((1u << bits) - 1u);
      word |= (uint32_t)sat_rte(col[c].f * (float)hi, 0, hi) << shift;
    }
    int es = oracle_elem_size(order, type);
    for (int b = 0; b < es; ++b) texel_out[b] = (uint8_t)(word >> (8 * b));
    return OR_SUCCESS;
  }
  int nc = oracle_channels(order), tb = type_bytes(type);
  for (int c = 0; c < nc; ++c) {
    val32 v = col[slot[c]];
    uint32_t code;
    switch (type) {
      case OR_UNORM_INT8: case OR_UNORM_INT16: case OR_SNORM_INT8: case OR_SNORM_INT16:
        code = (uint32_t)oracle_float_to_norm(type, v.f); break;
      case OR_HALF_FLOAT: code = oracle_float_to_half_rte(v.f); break;
      case OR_FLOAT: code = v.u; break;
      /* convert_char_sat / convert_short_sat of the int component */
      case OR_SIGNED_INT8: code = (uint32_t)(int32_t)clamp64(v.i, -128, 127); break;
      case OR_SIGNED_INT16: code = (uint32_t)(int32_t)clamp64(v.i, -32768, 32767); break;
      case OR_SIGNED_INT32: code = v.u; break;
      /* convert_uchar_sat / convert_ushort_sat of the uint component */
      case OR_UNSIGNED_INT8: code = v.u > 255u ? 255u : v.u; break;
      case OR_UNSIGNED_INT16: code = v.u > 65535u ? 65535u : v.u; break;
      default: code = v.u; break;
    }
    store_code(texel_out + c * tb, type, code);
  }
  return OR_SUCCESS;
}

int oracle_write_samples(oracle_image* img, int rtype, const int32_t* icoords,
                         int64_t cstride, const void* colors, int64_t n) {
  int es = oracle_elem_size(img->order, img->type);
  if (es < 0) return OR_IMAGE_FORMAT_NOT_SUPPORTED;
  if (rtype != rtype_of(img->type)) return OR_INVALID_OPERATION;
  for (int64_t s = 0; s < n; ++s) {
    const int32_t* ic = icoords + s * cstride;
    int nc = img->dims + (img->arrayed ? 1 : 0);  /* an array's layer is coordinate dims */
    int64_t i = ic[0], j = nc > 1 ? ic[1] : 0, k = nc > 2 ? ic[2] : 0;
    if (i < 0 || i >= img->width || j < 0 || j >= img->height || k < 0 || k >= img->depth)
      continue;                                              /* A15: no-op */
    uint8_t texel[16];
    oracle_convert_texel(img->order, img->type, rtype, (const uint8_t*)colors + 16 * s, texel);
    memcpy(img->data + k * img->slice_pitch + j * img->row_pitch + i * es, texel, (size_t)es);
  }
  return OR_SUCCESS;
}

/* ------------------------------------------------------------------ */
/* Bulk operations ([CL1.2 §5.2.2, §5.2.3, §5.3.3-5.3.5])               */
/* ------------------------------------------------------------------ */

/* clEnqueueCopyBufferRect: for z < region[2], y < region[1], x < region[0]:
 *   dst[dst_off + z*dsp + y*drp + x] = src[src_off + z*ssp + y*srp + x],
 *   *_off = origin[2]*slice_pitch + origin[1]*row_pitch + origin[0];
 * row_pitch 0 -> region[0]; slice_pitch 0 -> region[1]*row_pitch. */
void oracle_copy_rect(const uint8_t* src, uint8_t* dst, const size_t* so, const size_t* dso,
                      const size_t* region, size_t srp, size_t ssp, size_t drp, size_t dsp) {
  if (srp == 0) srp = region[0];
  if (ssp == 0) ssp = region[1] * srp;
  if (drp == 0) drp = region[0];
  if (dsp == 0) dsp = region[1] * drp;
  size_t soff = so[2] * ssp + so[1] * srp + so[0];
  size_t doff = dso[2] * dsp + dso[1] * drp + dso[0];
  for (size_t z = 0; z < region[2]; ++z)
    for (size_t y = 0; y < region[1]; ++y)
      for (size_t x = 0; x < region[0]; ++x)
        dst[doff + z * dsp + y * drp + x] = src[soff + z * ssp + y * srp + x];
}

/* clEnqueueFillBuffer: buf[offset + k] = pattern[k mod pattern_size], k < size. */
void oracle_fill_buffer(uint8_t* buf, const void* pattern, size_t pattern_size,
                        size_t offset, size_t size) {
  const uint8_t* p = (const uint8_t*)pattern;
  for (size_t k = 0; k < size; ++k) buf[offset + k] = p[k % pattern_size];
}

static uint8_t* texel_ptr(const oracle_image* img, size_t i, size_t j, size_t k) {
  int es = oracle_elem_size(img->order, img->type);
  return img->data + (int64_t)k * img->slice_pitch + (int64_t)j * img->row_pitch +
         (int64_t)i * es;
}

/* clEnqueueFillImage: fill_color converted once to one texel (reading A23),
 * replicated over the origin/region pixel box. */
int oracle_fill_image(oracle_image* img, int rtype, const void* color16,
                      const size_t* origin, const size_t* region) {
  uint8_t texel[16];
  int st = oracle_convert_texel(img->order, img->type, rtype, color16, texel);
  if (st != OR_SUCCESS) return st;
  int es = oracle_elem_size(img->order, img->type);
  for (size_t z = 0; z < region[2]; ++z)
    for (size_t y = 0; y < region[1]; ++y)
      for (size_t x = 0; x < region[0]; ++x)
        memcpy(texel_ptr(img, origin[0] + x, origin[1] + y, origin[2] + z), texel, (size_t)es);
  return OR_SUCCESS;
}

/* clEnqueueCopyImage: pixel box between images of the same format. */
void oracle_copy_image(const oracle_image* src, oracle_image* dst, const size_t* so,
                       const size_t* dso, const size_t* region) {
  int es = oracle_elem_size(src->order, src->type);
  for (size_t z = 0; z < region[2]; ++z)
    for (size_t y = 0; y < region[1]; ++y)
      for (size_t x = 0; x < region[0]; ++x)
        memcpy(texel_ptr(dst, dso[0] + x, dso[1] + y, dso[2] + z),
               texel_ptr(src, so[0] + x, so[1] + y, so[2] + z), (size_t)es);
}

/* clEnqueueCopyImageToBuffer: the pixel box, tightly packed at dst_offset. */
void oracle_copy_image_to_buffer(const oracle_image* src, uint8_t* dst, const size_t* so,
                                 const size_t* region, size_t dst_offset) {
  int es = oracle_elem_size(src->order, src->type);
  size_t n = 0;
  for (size_t z = 0; z < region[2]; ++z)
    for (size_t y = 0; y < region[1]; ++y)
      for (size_t x = 0; x < region[0]; ++x, ++n)
        memcpy(dst + dst_offset + n * (size_t)es, texel_ptr(src, so[0] + x, so[1] + y, so[2] + z),
               (size_t)es);
}

/* clEnqueueCopyBufferToImage: the inverse. */
void oracle_copy_buffer_to_image(const uint8_t* src, oracle_image* dst, size_t src_offset,
                                 const size_t* dso, const size_t* region) {
  int es = oracle_elem_size(dst->order, dst->type);
  size_t n = 0;
  for (size_t z = 0; z < region[2]; ++z)
    for (size_t y = 0; y < region[1]; ++y)
      for (size_t x = 0; x < region[0]; ++x, ++n)
        memcpy(texel_ptr(dst, dso[0] + x, dso[1] + y, dso[2] + z),
               src + src_offset + n * (size_t)es, (size_t)es);
}

/* clEnqueueReadImage / clEnqueueWriteImage ([CL1.2 §5.3.3]): host row_pitch
 * 0 -> region[0]*elem_size; slice_pitch 0 -> row_pitch*region[1].  For a 1D
 * image array region[1] counts layers and the host layers are slice_pitch
 * apart (0 -> row_pitch): "slice_pitch ... the size in bytes of ... each
 * image in a 1D or 2D image array ... calculated as row_pitch for a 1D image
 * array" -- so there the host row stride is slice_pitch. */
static void host_pitches(const oracle_image* img, const size_t* region, int es,
                         size_t* row_pitch, size_t* slice_pitch) {
  if (*row_pitch == 0) *row_pitch = region[0] * (size_t)es;
  if (img->arrayed && img->dims == 1) {
    if (*slice_pitch == 0) *slice_pitch = *row_pitch;
    *row_pitch = *slice_pitch;                  /* layer y at host + y*slice_pitch */
    *slice_pitch = *row_pitch * region[1];
    return;
  }
  if (*slice_pitch == 0) *slice_pitch = *row_pitch * region[1];
}

void oracle_read_image_rect(const oracle_image* img, const size_t* origin, const size_t* region,
                            size_t row_pitch, size_t slice_pitch, uint8_t* host) {
  int es = oracle_elem_size(img->order, img->type);
  host_pitches(img, region, es, &row_pitch, &slice_pitch);
  for (size_t z = 0; z < region[2]; ++z)
    for (size_t y = 0; y < region[1]; ++y)
      for (size_t x = 0; x < region[0]; ++x)
        memcpy(host + z * slice_pitch + y * row_pitch + x * (size_t)es,
               texel_ptr(img, origin[0] + x, origin[1] + y, origin[2] + z), (size_t)es);
}

void oracle_write_image_rect(oracle_image* img, const size_t* origin, const size_t* region,
                             size_t row_pitch, size_t slice_pitch, const uint8_t* host) {
  int es = oracle_elem_size(img->order, img->type);
  host_pitches(img, region, es, &row_pitch, &slice_pitch);
  for (size_t z = 0; z < region[2]; ++z)
    for (size_t y = 0; y < region[1]; ++y)
      for (size_t x = 0; x < region[0]; ++x)
        memcpy(texel_ptr(img, origin[0] + x, origin[1] + y, origin[2] + z),
               host + z * slice_pitch + y * row_pitch + x * (size_t)es, (size_t)es);
}

/* Pin P7: do the source and destination byte sets of a same-buffer rect copy
 * intersect?  Brute force over every pair of rows (each row is one contiguous
 * byte interval). */
int oracle_rect_overlap(const size_t* so, const size_t* dso, const size_t* region,
                        size_t srp, size_t ssp, size_t drp, size_t dsp) {
  if (srp == 0) srp = region[0];
  if (ssp == 0) ssp = region[1] * srp;
  if (drp == 0) drp = region[0];
  if (dsp == 0) dsp = region[1] * drp;
  size_t soff = so[2] * ssp + so[1] * srp + so[0];
  size_t doff = dso[2] * dsp + dso[1] * drp + dso[0];
  for (size_t z = 0; z < region[2]; ++z)
    for (size_t y = 0; y < region[1]; ++y) {
      size_t a0 = soff + z * ssp + y * srp, a1 = a0 + region[0];
      for (size_t z2 = 0; z2 < region[2]; ++z2)
        for (size_t y2 = 0; y2 < region[1]; ++y2) {
          size_t b0 = doff + z2 * dsp + y2 * drp, b1 = b0 + region[0];
          if (a0 < b1 && b0 < a1) return 1;
        }
    }
  return 0;
}
