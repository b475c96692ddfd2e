// validate.cpp -- pure host-side argument validation (no CUDA calls).
//
// Every enqueue of the runtime validates through these functions before it
// issues anything ("all validation happens before anything is enqueued").
// They are also exported (b2cl_ext.h) so the error behaviour is testable on
// a machine without a GPU.  Rules: [CL1.2 §5.2.2, §5.2.3, §5.3.1, §5.3.3,
// §5.5.1] with readings A5, A18, A21, A22 of DESIGN.md §3.
#include <stdint.h>

#include "internal.h"

namespace b2cl {

#define CHECK_ST(x)                      \
  do {                                   \
    cl_int _s = (x);                     \
    if (_s != CL_SUCCESS) return _s;     \
  } while (0)

// Khronos channel type / order -> internal codes (dev::TypeCode / OrderCode)
int type_code(cl_channel_type t) {
  switch (t) {
    case CL_SNORM_INT8: return dev::T_SNORM8;
    case CL_SNORM_INT16: return dev::T_SNORM16;
    case CL_UNORM_INT8: return dev::T_UNORM8;
    case CL_UNORM_INT16: return dev::T_UNORM16;
    case CL_SIGNED_INT8: return dev::T_SINT8;
    case CL_SIGNED_INT16: return dev::T_SINT16;
    case CL_SIGNED_INT32: return dev::T_SINT32;
    case CL_UNSIGNED_INT8: return dev::T_UINT8;
    case CL_UNSIGNED_INT16: return dev::T_UINT16;
    case CL_UNSIGNED_INT32: return dev::T_UINT32;
    case CL_HALF_FLOAT: return dev::T_HALF;
    case CL_FLOAT: return dev::T_FLOAT;
    case CL_UNORM_SHORT_565: return dev::T_U565;
    case CL_UNORM_SHORT_555: return dev::T_U555;
    case CL_UNORM_INT_101010: return dev::T_U101010;
    default: return -1;
  }
}

int order_code(cl_channel_order o) {
  switch (o) {
    case CL_R: return dev::O_R;
    case CL_A: return dev::O_A;
    case CL_RG: return dev::O_RG;
    case CL_RA: return dev::O_RA;
    case CL_RGBA: return dev::O_RGBA;
    case CL_BGRA: return dev::O_BGRA;
    case CL_ARGB: return dev::O_ARGB;
    case CL_INTENSITY: return dev::O_INTENSITY;
    case CL_LUMINANCE: return dev::O_LUMINANCE;
    case CL_RGB: return dev::O_RGB;
    case CL_RGBx: return dev::O_RGBX;
    default: return -1;  // CL_Rx, CL_RGx: not supported (reading A37)
  }
}

static bool known_type(cl_channel_type t) { return t >= 0x10D0 && t <= 0x10DE; }
static bool known_order(cl_channel_order o) { return o >= 0x10B0 && o <= 0x10BC; }

cl_int format_info(const cl_image_format* f, FormatInfo* out) {
  if (!f || !known_type(f->image_channel_data_type) || !known_order(f->image_channel_order))
    return CL_INVALID_IMAGE_FORMAT_DESCRIPTOR;
  const int t = type_code(f->image_channel_data_type);
  const int o = order_code(f->image_channel_order);
  if (t < 0 || o < 0) return CL_IMAGE_FORMAT_NOT_SUPPORTED;  // CL_Rx, CL_RGx (A37)
  // "CL_RGB or CL_RGBx: only if the channel data type is CL_UNORM_SHORT_565,
  // CL_UNORM_SHORT_555 or CL_UNORM_INT_101010" -- and those types need them
  const bool rgb = o == dev::O_RGB || o == dev::O_RGBX;
  if (rgb != dev::is_packed(t)) return CL_IMAGE_FORMAT_NOT_SUPPORTED;
  // [CL1.2 §5.3.1.1]: BGRA/ARGB only with 8-bit channels; INTENSITY and
  // LUMINANCE only with UNORM/SNORM 8/16, HALF and FLOAT.
  if (o == dev::O_BGRA || o == dev::O_ARGB) {
    if (!(t == dev::T_UNORM8 || t == dev::T_SNORM8 || t == dev::T_SINT8 || t == dev::T_UINT8))
      return CL_IMAGE_FORMAT_NOT_SUPPORTED;
  }
  if (o == dev::O_INTENSITY || o == dev::O_LUMINANCE) {
    if (!(t == dev::T_UNORM8 || t == dev::T_UNORM16 || t == dev::T_SNORM8 ||
          t == dev::T_SNORM16 || t == dev::T_HALF || t == dev::T_FLOAT))
      return CL_IMAGE_FORMAT_NOT_SUPPORTED;
  }
  out->type = t;
  out->order = o;
  out->nch = dev::order_channels(o);
  out->es = (size_t)dev::texel_bytes(t, o);
  out->rclass = dev::ret_class(t);
  return CL_SUCCESS;
}

static int image_dims(cl_mem_object_type t) {
  switch (t) {
    case CL_MEM_OBJECT_IMAGE1D:
    case CL_MEM_OBJECT_IMAGE1D_BUFFER: return 1;
    case CL_MEM_OBJECT_IMAGE2D:
    case CL_MEM_OBJECT_IMAGE1D_ARRAY: return 2;
    case CL_MEM_OBJECT_IMAGE3D:
    case CL_MEM_OBJECT_IMAGE2D_ARRAY: return 3;
    default: return 0;
  }
}

cl_int image_layout(const cl_image_format* fmt, const cl_image_desc* desc, ImageLayout* L) {
  FormatInfo fi;
  cl_int st = format_info(fmt, &fi);
  if (st != CL_SUCCESS) return st;
  if (!desc) return CL_INVALID_IMAGE_DESCRIPTOR;
  const cl_mem_object_type t = desc->image_type;
  const int dims = image_dims(t);
  if (dims == 0) return CL_INVALID_IMAGE_DESCRIPTOR;
  const bool arr1 = t == CL_MEM_OBJECT_IMAGE1D_ARRAY, arr2 = t == CL_MEM_OBJECT_IMAGE2D_ARRAY;
  const bool from_buffer = t == CL_MEM_OBJECT_IMAGE1D_BUFFER;
  if (desc->num_mip_levels != 0 || desc->num_samples != 0 ||
      (desc->buffer != nullptr) != from_buffer)
    return CL_INVALID_IMAGE_DESCRIPTOR;
  // storage extents: the layers of an array are its last storage axis
  size_t w = desc->image_width, h = 1, d = 1;
  if (arr1) h = desc->image_array_size;
  else if (dims > 1) h = desc->image_height;
  if (arr2) d = desc->image_array_size;
  else if (dims > 2) d = desc->image_depth;
  if (w == 0 || h == 0 || d == 0) return CL_INVALID_IMAGE_DESCRIPTOR;
  if (from_buffer) {
    if (w > kMaxBuffer) return CL_INVALID_IMAGE_SIZE;
  } else if (arr1 || arr2) {
    if (w > kMax2D || (arr1 ? h : d) > kMaxArray || (arr2 && h > kMax2D)) return CL_INVALID_IMAGE_SIZE;
  } else {
    const size_t maxw = dims == 3 ? kMax3D : kMax2D;
    if (w > maxw || h > maxw || d > kMax3D) return CL_INVALID_IMAGE_SIZE;
  }
  L->fmt = fi;
  L->dims = dims;
  L->arrayed = (arr1 || arr2) ? 1 : 0;
  L->w = w; L->h = h; L->d = d;
  // internal pitch (reading A21): rows 128-byte aligned -> every texel is
  // naturally aligned for its vector load, and TMA boxes are legal.  A 1D
  // image buffer is the buffer's bytes, tightly packed (one row).
  L->row_pitch = from_buffer ? w * fi.es : (w * fi.es + 127) / 128 * 128;
  L->slice_pitch = L->row_pitch * h;
  L->bytes = L->slice_pitch * d;
  return CL_SUCCESS;
}

bool tile_layout(ImageLayout* L) {
  if (L->dims != 2 || L->arrayed || L->fmt.es == 0 || L->fmt.es > 128 || (L->fmt.es & (L->fmt.es - 1))) return false;
  int sh = 0;
  while ((size_t)(1u << sh) * L->fmt.es < 128) ++sh;  // 2^sh texels per 128-byte tile row
  const size_t tiles_x = (L->w + (1u << sh) - 1) >> sh, bands = (L->h + 7) / 8;
  L->tiled = 1;
  L->tshift = sh;
  L->row_pitch = tiles_x * 1024;  // one band of 8 rows
  L->slice_pitch = L->row_pitch * bands;
  L->bytes = L->slice_pitch;
  return true;
}

// ---- rect copies ----
static bool rect_pitches(const size_t* region, size_t& rp, size_t& sp) {
  // pitch 0 -> defaults; a given pitch must be >= the default and the slice
  // pitch a multiple of the row pitch ([CL1.2 §5.2.2])
  if (rp == 0) rp = region[0];
  else if (rp < region[0]) return false;
  const unsigned __int128 min_sp = (unsigned __int128)region[1] * rp;
  if (min_sp >> 64) return false;
  if (sp == 0) sp = (size_t)min_sp;
  else if (sp < min_sp || sp % rp != 0) return false;
  return true;
}

// byte just past the box, or 0 on overflow
static unsigned __int128 box_end(const size_t* o, const size_t* region, size_t rp, size_t sp) {
  return (unsigned __int128)o[2] * sp + (unsigned __int128)o[1] * rp + o[0] +
         (unsigned __int128)(region[2] - 1) * sp + (unsigned __int128)(region[1] - 1) * rp +
         region[0];
}

static __int128 floor_div(__int128 a, __int128 b) {  // b > 0
  __int128 q = a / b;
  if ((a % b != 0) && (a < 0)) --q;
  return q;
}
static __int128 ceil_div(__int128 a, __int128 b) { return -floor_div(-a, b); }

// Exact test: rows are byte intervals [S + dz_s*sp + dy_s*rp, +R0); two rows
// meet iff |delta + dz*sp + dy*rp| < R0 with |dz| < R2, |dy| < R1.  For each
// dz the admissible dy form an interval, so the test is O(R2).
bool rect_overlap(const size_t* so, const size_t* dso, const size_t* region, size_t rp,
                  size_t sp) {
  const __int128 S = (__int128)so[2] * sp + (__int128)so[1] * rp + so[0];
  const __int128 D = (__int128)dso[2] * sp + (__int128)dso[1] * rp + dso[0];
  const __int128 R0 = region[0], R1 = region[1], R2 = region[2];
  const __int128 delta = S - D;
  for (__int128 dz = -(R2 - 1); dz <= R2 - 1; ++dz) {
    const __int128 x = delta + dz * (__int128)sp;
    __int128 lo = floor_div(-R0 - x, (__int128)rp) + 1;
    __int128 hi = ceil_div(R0 - x, (__int128)rp) - 1;
    if (lo < -(R1 - 1)) lo = -(R1 - 1);
    if (hi > R1 - 1) hi = R1 - 1;
    if (lo <= hi) return true;
  }
  return false;
}

cl_int validate_copy_rect(size_t src_size, size_t dst_size, bool same, const size_t* so,
                          const size_t* dso, const size_t* region, size_t& srp, size_t& ssp,
                          size_t& drp, size_t& dsp) {
  if (!so || !dso || !region) return CL_INVALID_VALUE;
  if (region[0] == 0 || region[1] == 0 || region[2] == 0) return CL_INVALID_VALUE;
  if (!rect_pitches(region, srp, ssp) || !rect_pitches(region, drp, dsp)) return CL_INVALID_VALUE;
  if (box_end(so, region, srp, ssp) > src_size) return CL_INVALID_VALUE;
  if (box_end(dso, region, drp, dsp) > dst_size) return CL_INVALID_VALUE;
  if (same) {
    if (srp != drp || ssp != dsp) return CL_INVALID_VALUE;  // reading A18: either differs
    if (rect_overlap(so, dso, region, srp, ssp)) return CL_MEM_COPY_OVERLAP;
  }
  return CL_SUCCESS;
}

cl_int validate_host_rect(size_t buf_size, const size_t* bo, const size_t* ho,
                          const size_t* region, size_t& brp, size_t& bsp, size_t& hrp,
                          size_t& hsp) {
  if (!bo || !ho || !region) return CL_INVALID_VALUE;
  if (region[0] == 0 || region[1] == 0 || region[2] == 0) return CL_INVALID_VALUE;
  if (!rect_pitches(region, brp, bsp) || !rect_pitches(region, hrp, hsp)) return CL_INVALID_VALUE;
  if (box_end(bo, region, brp, bsp) > buf_size) return CL_INVALID_VALUE;
  return CL_SUCCESS;
}

cl_int validate_fill_buffer(size_t buf_size, size_t ps, size_t offset, size_t size) {
  if (ps == 0 || ps > 128 || (ps & (ps - 1)) != 0) return CL_INVALID_VALUE;
  if (offset % ps != 0 || size % ps != 0) return CL_INVALID_VALUE;
  if (offset > buf_size || size > buf_size - offset) return CL_INVALID_VALUE;
  return CL_SUCCESS;
}

cl_int validate_sampler(cl_bool norm, cl_addressing_mode am, cl_filter_mode fm) {
  if (norm != CL_TRUE && norm != CL_FALSE) return CL_INVALID_VALUE;
  if (am < CL_ADDRESS_NONE || am > CL_ADDRESS_MIRRORED_REPEAT) return CL_INVALID_VALUE;
  if (fm != CL_FILTER_NEAREST && fm != CL_FILTER_LINEAR) return CL_INVALID_VALUE;
  if (!norm && (am == CL_ADDRESS_REPEAT || am == CL_ADDRESS_MIRRORED_REPEAT))
    return CL_INVALID_VALUE;  // reading A5
  return CL_SUCCESS;
}

cl_int validate_image_box(int dims, size_t w, size_t h, size_t d, const size_t* o,
                          const size_t* r) {
  if (!o || !r) return CL_INVALID_VALUE;
  if (r[0] == 0 || r[1] == 0 || r[2] == 0) return CL_INVALID_VALUE;
  if (dims < 3 && (o[2] != 0 || r[2] != 1)) return CL_INVALID_VALUE;
  if (dims < 2 && (o[1] != 0 || r[1] != 1)) return CL_INVALID_VALUE;
  if (o[0] > w || r[0] > w - o[0]) return CL_INVALID_VALUE;
  if (o[1] > h || r[1] > h - o[1]) return CL_INVALID_VALUE;
  if (o[2] > d || r[2] > d - o[2]) return CL_INVALID_VALUE;
  return CL_SUCCESS;
}

// ---- CUDA texture front end (reading A40) ----
cl_int channel_format(const b2cl_channel_format_desc* d, cl_image_format* f) {
  if (!d || !f) return CL_INVALID_VALUE;
  const int c[4] = {d->x, d->y, d->z, d->w}, b = d->x;
  int n = 0;
  while (n < 4 && c[n] != 0) ++n;
  for (int k = 0; k < 4; ++k)  // channels of one width, none after an empty one
    if ((k < n && c[k] != b) || (k >= n && c[k] != 0)) return CL_IMAGE_FORMAT_NOT_SUPPORTED;
  if (n != 1 && n != 2 && n != 4) return CL_IMAGE_FORMAT_NOT_SUPPORTED;
  f->image_channel_order = n == 1 ? CL_R : (n == 2 ? CL_RG : CL_RGBA);
  switch (d->kind) {
    case B2CL_CHANNEL_SIGNED:
      if (b == 8) f->image_channel_data_type = CL_SIGNED_INT8;
      else if (b == 16) f->image_channel_data_type = CL_SIGNED_INT16;
      else if (b == 32) f->image_channel_data_type = CL_SIGNED_INT32;
      else return CL_IMAGE_FORMAT_NOT_SUPPORTED;
      return CL_SUCCESS;
    case B2CL_CHANNEL_UNSIGNED:
      if (b == 8) f->image_channel_data_type = CL_UNSIGNED_INT8;
      else if (b == 16) f->image_channel_data_type = CL_UNSIGNED_INT16;
      else if (b == 32) f->image_channel_data_type = CL_UNSIGNED_INT32;
      else return CL_IMAGE_FORMAT_NOT_SUPPORTED;
      return CL_SUCCESS;
    case B2CL_CHANNEL_FLOAT:
      if (b == 16) f->image_channel_data_type = CL_HALF_FLOAT;
      else if (b == 32) f->image_channel_data_type = CL_FLOAT;
      else return CL_IMAGE_FORMAT_NOT_SUPPORTED;
      return CL_SUCCESS;
    default: return CL_IMAGE_FORMAT_NOT_SUPPORTED;
  }
}

cl_int texture_mapping(const b2cl_texture_desc* td, cl_uint dims, const cl_image_format* stored,
                       cl_image_format* view, cl_bool* norm, cl_addressing_mode* am,
                       cl_filter_mode* fm, b2cl_rtype* rt) {
  if (!td || !stored || dims < 1 || dims > 3) return CL_INVALID_VALUE;
  FormatInfo fi;
  CHECK_ST(format_info(stored, &fi));
  // a CUDA texture has 1, 2 or 4 channels in memory order, no packed words
  if (fi.order != dev::O_R && fi.order != dev::O_RG && fi.order != dev::O_RGBA)
    return CL_IMAGE_FORMAT_NOT_SUPPORTED;
  // stored channel: signedness and width (UNORM / UNSIGNED_INT alike)
  const int t = fi.type;
  const bool is_float = t == dev::T_HALF || t == dev::T_FLOAT;
  const bool sgn = t == dev::T_SNORM8 || t == dev::T_SNORM16 || t == dev::T_SINT8 ||
                   t == dev::T_SINT16 || t == dev::T_SINT32;
  const int bits = 8 * dev::type_bytes(t);
  cl_channel_type vt;
  if (td->read_mode == B2CL_READ_NORMALIZED_FLOAT) {
    if (is_float || bits == 32) return CL_INVALID_VALUE;  // 8- and 16-bit integers only
    vt = bits == 8 ? (sgn ? CL_SNORM_INT8 : CL_UNORM_INT8) : (sgn ? CL_SNORM_INT16 : CL_UNORM_INT16);
  } else if (td->read_mode == B2CL_READ_ELEMENT_TYPE) {
    if (t == dev::T_HALF) vt = CL_HALF_FLOAT;
    else if (t == dev::T_FLOAT) vt = CL_FLOAT;
    else if (bits == 8) vt = sgn ? CL_SIGNED_INT8 : CL_UNSIGNED_INT8;
    else if (bits == 16) vt = sgn ? CL_SIGNED_INT16 : CL_UNSIGNED_INT16;
    else vt = sgn ? CL_SIGNED_INT32 : CL_UNSIGNED_INT32;
  } else {
    return CL_INVALID_VALUE;
  }
  // one OpenCL sampler for all axes: the sampled axes' modes must agree
  const cl_uint m = td->address_mode[0];
  for (cl_uint d = 0; d < dims; ++d)
    if (td->address_mode[d] != m) return CL_INVALID_VALUE;
  cl_addressing_mode a;
  switch (m) {
    case B2CL_TEX_WRAP: a = CL_ADDRESS_REPEAT; break;
    case B2CL_TEX_CLAMP: a = CL_ADDRESS_CLAMP_TO_EDGE; break;
    case B2CL_TEX_MIRROR: a = CL_ADDRESS_MIRRORED_REPEAT; break;
    case B2CL_TEX_BORDER: a = CL_ADDRESS_CLAMP; break;
    default: return CL_INVALID_VALUE;
  }
  if (td->filter_mode != B2CL_TEX_POINT && td->filter_mode != B2CL_TEX_LINEAR) return CL_INVALID_VALUE;
  for (int c = 0; c < 4; ++c)
    if (td->border_color[c] != 0.0f) return CL_INVALID_VALUE;
  const cl_bool nc = td->normalized_coords ? CL_TRUE : CL_FALSE;
  const cl_filter_mode f = td->filter_mode == B2CL_TEX_LINEAR ? CL_FILTER_LINEAR : CL_FILTER_NEAREST;
  CHECK_ST(validate_sampler(nc, a, f));  // wrap / mirror need normalized coordinates (A5)
  const b2cl_rtype r = dev::ret_class(type_code(vt));
  // "linear filtering ... only for textures configured to return floating-point data"
  if (f == CL_FILTER_LINEAR && r != B2CL_RTYPE_FLOAT) return CL_INVALID_OPERATION;
  if (view) {
    view->image_channel_order = stored->image_channel_order;
    view->image_channel_data_type = vt;
  }
  if (norm) *norm = nc;
  if (am) *am = a;
  if (fm) *fm = f;
  if (rt) *rt = r;
  return CL_SUCCESS;
}

bool image_boxes_overlap(const size_t* a, const size_t* b, const size_t* r) {
  for (int k = 0; k < 3; ++k)
    if (!(a[k] < b[k] + r[k] && b[k] < a[k] + r[k])) return false;
  return true;
}

}  // namespace b2cl

// ---------------------------------------------------------------- exports
using namespace b2cl;

extern "C" cl_int b2clValidateCopyBufferRect(size_t src_size, size_t dst_size, cl_int same_buffer,
                                             const size_t* so, const size_t* dso,
                                             const size_t* region, size_t srp, size_t ssp,
                                             size_t drp, size_t dsp) {
  return validate_copy_rect(src_size, dst_size, same_buffer != 0, so, dso, region, srp, ssp, drp,
                            dsp);
}

extern "C" cl_int b2clRectOverlap(const size_t* so, const size_t* dso, const size_t* region,
                                  size_t rp, size_t sp) {
  if (!so || !dso || !region || region[0] == 0 || region[1] == 0 || region[2] == 0) return 0;
  size_t r = rp, s = sp;
  if (!rect_pitches(region, r, s)) return 0;
  return rect_overlap(so, dso, region, r, s) ? 1 : 0;
}

extern "C" cl_int b2clValidateFillBuffer(size_t buffer_size, size_t pattern_size, size_t offset,
                                         size_t size) {
  return validate_fill_buffer(buffer_size, pattern_size, offset, size);
}

extern "C" cl_int b2clTextureMapping(const b2cl_texture_desc* td, cl_uint dims,
                                     const cl_image_format* stored, cl_image_format* view,
                                     cl_bool* norm, cl_addressing_mode* am, cl_filter_mode* fm,
                                     b2cl_rtype* rt) {
  return texture_mapping(td, dims, stored, view, norm, am, fm, rt);
}

extern "C" cl_int b2clChannelFormat(const b2cl_channel_format_desc* d, cl_image_format* f) {
  return channel_format(d, f);
}

extern "C" cl_int b2clValidateSampler(cl_bool normalized_coords, cl_addressing_mode am,
                                      cl_filter_mode fm) {
  return validate_sampler(normalized_coords, am, fm);
}

extern "C" cl_int b2clImageLayout(const cl_image_format* fmt, const cl_image_desc* desc,
                                  size_t* elem_size, size_t* row_pitch, size_t* slice_pitch,
                                  size_t* total_bytes) {
  ImageLayout L;
  cl_int st = image_layout(fmt, desc, &L);
  if (st != CL_SUCCESS) return st;
  if (elem_size) *elem_size = L.fmt.es;
  if (row_pitch) *row_pitch = L.row_pitch;
  if (slice_pitch) *slice_pitch = L.slice_pitch;
  if (total_bytes) *total_bytes = L.bytes;
  return CL_SUCCESS;
}

extern "C" cl_int b2clValidateImageBox(cl_mem_object_type image_type, size_t width, size_t height,
                                       size_t depth, const size_t* origin, const size_t* region) {
  const int dims = image_type == CL_MEM_OBJECT_IMAGE1D   ? 1
                   : image_type == CL_MEM_OBJECT_IMAGE2D ? 2
                   : image_type == CL_MEM_OBJECT_IMAGE3D ? 3
                                                         : 0;
  if (!dims) return CL_INVALID_MEM_OBJECT;
  return validate_image_box(dims, width, dims > 1 ? height : 1, dims > 2 ? depth : 1, origin,
                            region);
}
