// internal.h -- host runtime internals of libb2cl (not part of the C-ABI).
#pragma once
#include <stddef.h>
#include <stdint.h>

#include "../../../include/b2cl_cl.h"
#include "../../../include/b2cl_ext.h"
#include "../device/codes.h"

namespace b2cl {

constexpr size_t kMax2D = 65536;  // CL_DEVICE_IMAGE2D_MAX_WIDTH/HEIGHT (and 1D width)
constexpr size_t kMax3D = 16384;  // CL_DEVICE_IMAGE3D_MAX_*
constexpr size_t kMaxArray = 65536;            // CL_DEVICE_IMAGE_MAX_ARRAY_SIZE
constexpr size_t kMaxBuffer = (1ull << 31) - 1;  // CL_DEVICE_IMAGE_MAX_BUFFER_SIZE (texels):
                                                 // the int coordinate's range, not a texture limit

struct FormatInfo {
  int type, order, nch, rclass;  // dev::TypeCode, dev::OrderCode, channels, dev::RetCode
  size_t es;                     // elem_size
};

// Storage view of every image type.  `dims` counts STORAGE axes: an image
// array keeps its layers on the axis after the sampled ones -- a 1D image
// array is stored as a w x layers 2D image (dims 2, arrayed), a 2D image
// array as a w x h x layers 3D image (dims 3, arrayed) -- so every pixel-box
// operation (copies, fills, host transfers) addresses it as that image, with
// origin/region[1] (1D array) or [2] (2D array) selecting layers as
// [CL1.2 §5.3.3] specifies.  Sampling uses dims - arrayed axes plus the layer.
struct ImageLayout {
  FormatInfo fmt;
  int dims;
  int arrayed;  // 1 for CL_MEM_OBJECT_IMAGE1D_ARRAY / IMAGE2D_ARRAY
  size_t w, h, d;
  size_t row_pitch, slice_pitch, bytes;
  // tiled storage (B2CL_MEM_TILED_IMAGE): 1 KiB tiles of 8 rows x 128 B;
  // row_pitch is then the bytes of one band of 8 rows, slice_pitch the total
  int tiled = 0, tshift = 0;
};

// turn a 2D image layout into the tiled one (false: not a tileable image)
bool tile_layout(ImageLayout* L);

int type_code(cl_channel_type t);
int order_code(cl_channel_order o);
cl_int format_info(const cl_image_format* f, FormatInfo* out);
cl_int image_layout(const cl_image_format* fmt, const cl_image_desc* desc, ImageLayout* L);
bool rect_overlap(const size_t* so, const size_t* dso, const size_t* region, size_t rp, size_t sp);
cl_int validate_copy_rect(size_t src_size, size_t dst_size, bool same, const size_t* so,
                          const size_t* dso, const size_t* region, size_t& srp, size_t& ssp,
                          size_t& drp, size_t& dsp);
cl_int validate_host_rect(size_t buf_size, const size_t* bo, const size_t* ho,
                          const size_t* region, size_t& brp, size_t& bsp, size_t& hrp,
                          size_t& hsp);
cl_int validate_fill_buffer(size_t buf_size, size_t ps, size_t offset, size_t size);
cl_int validate_sampler(cl_bool norm, cl_addressing_mode am, cl_filter_mode fm);
cl_int validate_image_box(int dims, size_t w, size_t h, size_t d, const size_t* o,
                          const size_t* r);
bool image_boxes_overlap(const size_t* a, const size_t* b, const size_t* r);
cl_int channel_format(const b2cl_channel_format_desc* d, cl_image_format* f);
cl_int texture_mapping(const b2cl_texture_desc* td, cl_uint dims, const cl_image_format* stored,
                       cl_image_format* view, cl_bool* norm, cl_addressing_mode* am,
                       cl_filter_mode* fm, b2cl_rtype* rt);

}  // namespace b2cl
