// codes.h -- internal format / sampler codes and the device image descriptor,
// shared by the kernels and the host runtime of libb2cl (not by oracle/).
#pragma once
#include <stdint.h>

#ifdef __CUDACC__
#define B2CL_HD __host__ __device__
#else
#define B2CL_HD
#endif

namespace b2cl {
namespace dev {

// ---- internal format codes (host maps the Khronos enums onto these) ----
enum TypeCode : int {
  T_SNORM8 = 0, T_SNORM16, T_UNORM8, T_UNORM16, T_SINT8, T_SINT16, T_SINT32,
  T_UINT8, T_UINT16, T_UINT32, T_HALF, T_FLOAT,
  // packed normalized RGB words ([CL1.2 §5.3.1.1]), orders O_RGB / O_RGBX only
  T_U565, T_U555, T_U101010, T_COUNT
};
enum OrderCode : int {
  O_R = 0, O_A, O_RG, O_RA, O_RGBA, O_BGRA, O_ARGB, O_INTENSITY, O_LUMINANCE, O_RGB, O_RGBX,
  O_COUNT
};
enum AddrCode : int { A_NONE = 0, A_CTE, A_CLAMP, A_REPEAT, A_MIRROR };
enum FiltCode : int { F_NEAREST = 0, F_LINEAR = 1 };
enum RetCode : int { R_F = 0, R_I = 1, R_UI = 2 };
constexpr int RT = -1;  // "decided at run time" template value

struct Image {            // the CLImage of Fig. 6, device view
  char* ptr;
  int w, h, d;            // unused dimensions are 1 (global extent for a shard)
  int type, order;        // TypeCode / OrderCode
  int es, nch;            // elem_size, channels
  uint64_t rp, sp;        // row_pitch, slice_pitch (bytes)
  // Outer axis (rows of a 2D image, slices of a 3D image) as stored: storage
  // row s holds global index (ob + s) mod (outer extent), s < os.  A plain
  // image has ob = 0 and os = its extent; a shard (b2clCreateImageShard)
  // stores its band plus halo rows of a larger global image.
  int ob, os;
  // Tiled storage (B2CL_MEM_TILED_IMAGE, 2D images): 1 KiB tiles of 8 rows x
  // 128 bytes (2^tshift texels); rp is then the bytes of one band of 8 rows
  // (tiles_x KiB), and texel (i, j) lives at
  //   ptr + (j >> 3) * rp + (i >> tshift) * 1024 + (j & 7) * 128 + (i & (2^tshift - 1)) * es.
  int tiled, tshift;
};

struct Sampler {
  int norm, addr, filt;
};

B2CL_HD constexpr bool is_packed(int t) { return t == T_U565 || t == T_U555 || t == T_U101010; }
// bytes of one channel (a packed type: of the whole word)
B2CL_HD constexpr int type_bytes(int t) {
  return (t == T_SNORM8 || t == T_UNORM8 || t == T_SINT8 || t == T_UINT8)   ? 1
         : (t == T_SINT32 || t == T_UINT32 || t == T_FLOAT || t == T_U101010) ? 4
                                                                              : 2;
}
B2CL_HD constexpr int order_channels(int o) {
  return (o == O_R || o == O_A || o == O_INTENSITY || o == O_LUMINANCE) ? 1
         : (o == O_RG || o == O_RA)                                   ? 2
         : (o == O_RGB || o == O_RGBX)                                ? 3
                                                                      : 4;
}
// element size (CLImage.elem_size, Fig. 6): channels x channel bytes, or the packed word
B2CL_HD constexpr int texel_bytes(int t, int o) {
  return is_packed(t) ? type_bytes(t) : order_channels(o) * type_bytes(t);
}
B2CL_HD constexpr int ret_class(int t) {
  return (t == T_SINT8 || t == T_SINT16 || t == T_SINT32)    ? R_I
         : (t == T_UINT8 || t == T_UINT16 || t == T_UINT32) ? R_UI
                                                            : R_F;
}

}  // namespace dev
}  // namespace b2cl
