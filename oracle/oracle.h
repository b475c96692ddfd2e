/*
 * oracle.h -- CPU oracle for the OpenCL 1.2 image / sampler / memory-object
 * rules that the b2cl hot path emulates on B200.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py (cpu_baseline leg and --impl reference) may load this library.
 * The product path (paper_conf_sc_kimdjjl15_b200/) never links, imports or
 * calls anything here, and this file shares no header, table or helper with
 * it.  Enum values are restated here from the public Khronos cl.h.
 *
 * What the paper fixes (PAPER.md, cited as P:<line>):
 *   - an image object is a CUDA memory object plus {format, desc, row_pitch,
 *     slice_pitch, elem_size, channels}          (Fig. 6)
 *   - "We support all OpenCL image-related functions" and read_imageX /
 *     write_imageX read and write through that pointer
 *   - the image features are channel description, normalized coordinates,
 *     addressing mode and filter mode
 * Everything numeric is therefore the OpenCL 1.2 specification's
 * ([CL1.2 §8.1-8.3, §6.12.14, §5.2.2-5.3.5]); each function below names the
 * rule it follows, and DESIGN.md §3 lists every reading taken where the
 * spec is silent (A1..A33 of SURVEY.md §8(c)).
 *
 * Arithmetic discipline: every fp32 operation in the address path is one
 * IEEE round-to-nearest operation in the written order (compiled with
 * -ffp-contract=off, no fast-math).  The LINEAR blend is evaluated in fp64
 * and rounded once to fp32 (reading A10/O6).
 */
#ifndef B2CL_ORACLE_H
#define B2CL_ORACLE_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- Khronos enum values, restated (public cl.h) ---- */
#define OR_R          0x10B0
#define OR_A          0x10B1
#define OR_RG         0x10B2
#define OR_RA         0x10B3
#define OR_RGB        0x10B4
#define OR_RGBA       0x10B5
#define OR_BGRA       0x10B6
#define OR_ARGB       0x10B7
#define OR_INTENSITY  0x10B8
#define OR_LUMINANCE  0x10B9
#define OR_Rx         0x10BA   /* not supported (reading A37) */
#define OR_RGx        0x10BB   /* not supported (reading A37) */
#define OR_RGBx       0x10BC

#define OR_SNORM_INT8      0x10D0
#define OR_SNORM_INT16     0x10D1
#define OR_UNORM_INT8      0x10D2
#define OR_UNORM_INT16     0x10D3
#define OR_UNORM_SHORT_565  0x10D4  /* packed: R 15:11, G 10:5, B 4:0 (CL_RGB / CL_RGBx) */
#define OR_UNORM_SHORT_555  0x10D5  /* packed: x 15, R 14:10, G 9:5, B 4:0 */
#define OR_UNORM_INT_101010 0x10D6  /* packed: x 31:30, R 29:20, G 19:10, B 9:0 */
#define OR_SIGNED_INT8     0x10D7
#define OR_SIGNED_INT16    0x10D8
#define OR_SIGNED_INT32    0x10D9
#define OR_UNSIGNED_INT8   0x10DA
#define OR_UNSIGNED_INT16  0x10DB
#define OR_UNSIGNED_INT32  0x10DC
#define OR_HALF_FLOAT      0x10DD
#define OR_FLOAT           0x10DE

#define OR_ADDRESS_NONE             0x1130
#define OR_ADDRESS_CLAMP_TO_EDGE    0x1131
#define OR_ADDRESS_CLAMP            0x1132
#define OR_ADDRESS_REPEAT           0x1133
#define OR_ADDRESS_MIRRORED_REPEAT  0x1134
#define OR_FILTER_NEAREST           0x1140
#define OR_FILTER_LINEAR            0x1141

/* return type of the read/write built-in: read_imagef / read_imagei / read_imageui */
#define OR_RT_F   0
#define OR_RT_I   1
#define OR_RT_UI  2

/* status codes (Khronos values) */
#define OR_SUCCESS                 0
#define OR_INVALID_VALUE         (-30)
#define OR_INVALID_OPERATION     (-59)
#define OR_IMAGE_FORMAT_NOT_SUPPORTED (-10)

/* An image as the oracle sees it: texel (i,j,k) lives at
 * data + k*slice_pitch + j*row_pitch + i*elem_size   (Fig. 6 fields).
 * Image arrays ([CL1.2 §5.3.1], §8.4): `arrayed` = 1 and `dims` is the number
 * of SAMPLED axes; the layer is the next axis -- a 1D image array of L layers
 * is width x L (j = layer, row_pitch = bytes per layer), a 2D image array is
 * width x height x L (k = layer, slice_pitch = bytes per layer).  A 1D image
 * buffer is a plain dims = 1 image over the buffer's bytes. */
typedef struct {
  uint8_t* data;
  int64_t width, height, depth;   /* unused dimensions are 1 */
  int64_t row_pitch, slice_pitch; /* bytes */
  int32_t dims;                   /* sampled axes: 1, 2 or 3 */
  uint32_t order, type;
  int32_t arrayed;                /* 0, or 1 for a 1D / 2D image array */
} oracle_image;

/* bytes per element, or -1 if (order,type) is not an in-scope format */
int oracle_elem_size(uint32_t order, uint32_t type);
int oracle_channels(uint32_t order);

/* ---- single-channel conversions (exposed for the P4 exhaustive pins) ---- */
float    oracle_half_to_float(uint16_t h);
uint16_t oracle_float_to_half_rte(float f);
/* read conversion of one stored channel code to float ([CL1.2 §8.3.1]) */
float    oracle_norm_to_float(uint32_t type, int32_t code);
/* write conversion of one float to a stored channel code ([CL1.2 §8.3.1.1]) */
int32_t  oracle_float_to_norm(uint32_t type, float f);

/* ---- sampler addressing for one axis ([CL1.2 §8.2]) ----
 * nearest: *i0 = index (may be out of range -> border); linear: i0,i1,a. */
void oracle_axis_nearest(float s, int64_t n, int normalized, uint32_t addressing,
                         int64_t* i0);
void oracle_axis_linear(float s, int64_t n, int normalized, uint32_t addressing,
                        int64_t* i0, int64_t* i1, float* a);

/* ---- image-array layer selection ([CL1.2 §8.4]) ----
 * layer = clamp(rint(c), 0, n - 1), rint = round half to even; NaN -> 0
 * (reading A35).  The layer coordinate is never normalized or filtered. */
int64_t oracle_layer_index(float c, int64_t n);

/* ---- the read built-ins ----
 * coord: dims (+1 for an array: the layer) floats (1D: s, 2D: s,t, 3D: s,t,r;
 * 1D array: s,layer; 2D array: s,t,layer).  out: 16 bytes
 * (float4 / int4 / uint4).  Returns OR_SUCCESS or a Khronos error for
 * combinations the readings A5/A6/A7 reject. */
int oracle_read_image(const oracle_image* img, int normalized, uint32_t addressing,
                      uint32_t filter, int rtype, const float* coord, void* out16);
/* integer-coordinate form (reading A30): unnormalized, NEAREST, non-wrapping. */
int oracle_read_image_icoord(const oracle_image* img, int normalized, uint32_t addressing,
                             uint32_t filter, int rtype, const int32_t* icoord, void* out16);

/* n samples; coords are packed with stride cstride floats (or int32s when
 * coord_is_int) per sample; out is n x 16 bytes. */
int oracle_read_samples(const oracle_image* img, int normalized, uint32_t addressing,
                        uint32_t filter, int rtype, int coord_is_int, const void* coords,
                        int64_t cstride, int64_t n, void* out);

/* Grid mode (the b2clEnqueueReadImageGrid extension): output element
 * (x,y,z) samples at coord[k] = (((A[4k]*x + A[4k+1]*y) + A[4k+2]*z) + A[4k+3]),
 * each operation one fp32 RN op in that order, for k < dims.  Only the rows
 * y in [y0,y1) of slices z in [z0,z1) are produced, tightly packed as
 * [z-z0][y-y0][x][c] with c < out_channels, 4 bytes per channel.
 * nthreads > 1 splits the rows across pthreads (no other change). */
int oracle_read_grid(const oracle_image* img, int normalized, uint32_t addressing,
                     uint32_t filter, int rtype, const float* affine12,
                     int64_t out_w, int64_t out_h, int64_t out_d, int out_channels,
                     int64_t z0, int64_t z1, int64_t y0, int64_t y1,
                     void* out, int nthreads);

/* ---- the write built-ins ([CL1.2 §6.12.14.4, §8.3]) ----
 * icoords: stride cstride int32 per sample; colors: n x 16 bytes.
 * Out-of-range coordinates are no-ops (reading A15). */
int oracle_write_samples(oracle_image* img, int rtype, const int32_t* icoords,
                         int64_t cstride, const void* colors, int64_t n);
/* Convert one color to one texel's bytes (used by FillImage, [CL1.2 §5.3.4]). */
int oracle_convert_texel(uint32_t order, uint32_t type, int rtype, const void* color16,
                         uint8_t* texel_out);

/* ---- CUDA texture fetches (NEXT row 3: the CUDA side of the paper's
 * CUDA-to-OpenCL texture translation) ----
 * A CUDA texture over the texels of `img` (order R, RG or RGBA = a 1-, 2- or
 * 4-channel CUDA array or linear memory), fetched as the CUDA C Programming
 * Guide's "Texture Fetching" appendix defines ([CUDA-PG TF]).  img->type only
 * says how a channel is STORED -- its bits and signedness (UNORM and
 * UNSIGNED_INT alike are unsigned integers, SNORM and SIGNED_INT signed,
 * HALF_FLOAT / FLOAT floating point); read_mode decides the conversion.
 * out16: the fetched vector as float4 / int4 / uint4 bits, components beyond
 * the channel count 0.  Returns OR_INVALID_VALUE for what CUDA does not
 * support (wrap/mirror with unnormalized coordinates, a normalized-float read
 * of a 32-bit or floating-point channel) and OR_INVALID_OPERATION for linear
 * filtering of an element-type integer read. */
typedef struct {
  uint32_t address_mode[3];  /* cudaTextureAddressMode: 0 wrap, 1 clamp, 2 mirror, 3 border */
  uint32_t filter_mode;      /* cudaTextureFilterMode: 0 point, 1 linear */
  uint32_t read_mode;        /* cudaTextureReadMode: 0 element type, 1 normalized float */
  int32_t normalized_coords;
} oracle_tex_desc;

/* tex1D / tex2D / tex3D (coord: dims floats) and tex1DLayered / tex2DLayered
 * (img->arrayed; coord: dims floats then the integer layer as a float). */
int oracle_tex_fetch(const oracle_image* img, const oracle_tex_desc* td, const float* coord,
                     void* out16);
/* tex1Dfetch on linear memory: the texel at integer index x, 0 out of range. */
int oracle_tex1Dfetch(const oracle_image* img, uint32_t read_mode, int32_t x, void* out16);

/* ---- bulk runtime operations ([CL1.2 §5.2.2-5.3.5]) ----
 * All origins/regions are size_t[3]; rect pitches 0 take the spec defaults. */
void oracle_copy_rect(const uint8_t* src, uint8_t* dst, const size_t* src_origin,
                      const size_t* dst_origin, const size_t* region,
                      size_t src_row_pitch, size_t src_slice_pitch,
                      size_t dst_row_pitch, size_t dst_slice_pitch);
void oracle_fill_buffer(uint8_t* buf, const void* pattern, size_t pattern_size,
                        size_t offset, size_t size);
int  oracle_fill_image(oracle_image* img, int rtype, const void* color16,
                       const size_t* origin, const size_t* region);
void oracle_copy_image(const oracle_image* src, oracle_image* dst,
                       const size_t* src_origin, const size_t* dst_origin,
                       const size_t* region);
void oracle_copy_image_to_buffer(const oracle_image* src, uint8_t* dst,
                                 const size_t* src_origin, const size_t* region,
                                 size_t dst_offset);
void oracle_copy_buffer_to_image(const uint8_t* src, oracle_image* dst,
                                 size_t src_offset, const size_t* dst_origin,
                                 const size_t* region);
/* Read/WriteImage against host memory with host pitches (0 = tight). */
void oracle_read_image_rect(const oracle_image* img, const size_t* origin,
                            const size_t* region, size_t row_pitch, size_t slice_pitch,
                            uint8_t* host);
void oracle_write_image_rect(oracle_image* img, const size_t* origin, const size_t* region,
                             size_t row_pitch, size_t slice_pitch, const uint8_t* host);
/* Brute-force byte-set overlap of a same-buffer rect copy (pin P7). */
int  oracle_rect_overlap(const size_t* src_origin, const size_t* dst_origin,
                         const size_t* region, size_t src_row_pitch, size_t src_slice_pitch,
                         size_t dst_row_pitch, size_t dst_slice_pitch);

#ifdef __cplusplus
}
#endif
#endif
