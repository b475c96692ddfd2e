// launch.h -- host-side launchers of the b2cl kernels (internal to libb2cl.so).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../device/codes.h"

namespace b2cl {

enum CoordMode : int { COORD_GRID = 0, COORD_LIST_F = 1, COORD_LIST_I = 2 };

struct SampleParams {
  dev::Image im;
  dev::Sampler smp;
  int rclass;       // dev::RetCode
  int dims;         // sampled axes 1..3
  int arr;          // 1: image array; coordinate `dims` selects the layer ([CL1.2 §8.4])
  float A[12];      // grid: affine coordinate map
  int ow, oh, od;   // grid: output region dims
  int ox, oy, oz;   // grid: output region origin (coordinates use origin + index)
  int outc;         // grid: output channels 1..4
  const char* coords;  // list: coordinates (already offset)
  uint64_t n;          // list: number of samples
  char* out;           // output (already offset)
};

struct RectParams {
  const char* src;   // COPY: source at origin
  char* dst;         // destination at origin
  uint64_t R0;       // bytes per row
  uint32_t R1, R2;   // rows, slices
  uint64_t srp, ssp, drp, dsp;
  uint32_t ptile[32];     // FILL: 128-byte tile (pattern repeated)
  uint32_t color[4];      // FILL_IMAGE: color bits
  int type, order, es;    // FILL_IMAGE: format
  // set by launch_rect: rows = R1*R2, row_step = rows walked per loop
  // iteration of a thread, step_dz / step_dy = row_step as (slices, rows)
  uint64_t rows, row_step;
  uint32_t step_dz, step_dy;
};

struct WriteParams {
  dev::Image im;
  int rclass, dims;
  const int32_t* coords;  // n x {1,2,4}
  const uint32_t* colors; // n x 4
  uint64_t n;
};

enum RectMode : int { RECT_COPY = 0, RECT_FILL = 1, RECT_FILL_IMAGE = 2, RECT_COPY_ALIGNED = 3 };

// Texel-addressed box copy / fill for TILED images (B2CL_MEM_TILED_IMAGE):
// each side is pitched-linear or tiled (dev::Image::tiled); one thread per
// texel moves es bytes (or writes the fill colour converted with the
// write_image rules).  Used for every pixel-box operation that touches a
// tiled image: Copy{Image,ImageToBuffer,BufferToImage}, FillImage, the
// host transfers (through a linear staging buffer) and the upload at creation.
struct TexSide {
  char* ptr;        // texel (0,0,0) of the box (linear) or the image base (tiled)
  uint64_t rp, sp;  // linear: row / slice pitch; tiled: rp = bytes of a band of 8 rows
  int tiled, tshift;
  int ox, oy;       // tiled: the box origin (texels, rows)
};
struct TexCopyParams {
  TexSide src, dst;
  uint32_t w, h, d;     // box (texels)
  int es;               // element size
  int fill;             // 1: write the colour below instead of copying
  uint32_t color[4];
  int type, order;      // fill: the format (dev::TypeCode, OrderCode)
};
cudaError_t launch_texcopy(const TexCopyParams& p, cudaStream_t stream);

// Each launcher enqueues exactly one kernel (or none for empty work) on
// `stream` and returns the launch status.
cudaError_t launch_sample(const SampleParams& p, int coord_mode, cudaStream_t stream);
cudaError_t launch_rect(RectParams& p, int mode, cudaStream_t stream);
cudaError_t launch_write(const WriteParams& p, cudaStream_t stream);
// config-3 TMA-staged trilinear kernel (sample_vol.cu); *used = false when
// the call does not qualify (nothing enqueued)
cudaError_t launch_sample_vol(const SampleParams& p, cudaStream_t stream, bool* used);
// ... and its rotated-map variant (x, y any affine in the output x, y; z separable)
cudaError_t launch_sample_volr(const SampleParams& p, cudaStream_t stream, bool* used);

// ... and 2D RGBA32F LINEAR reads under any affine map (sample_box.cu)
cudaError_t launch_sample_box(const SampleParams& p, cudaStream_t stream, bool* used);

// count of kernels launched by this library; the name of the last kernel this
// host thread launched (b2clGetLastKernelName: the bench reports it)
uint64_t launch_count();
void count_launch(const char* kernel);
const char* last_kernel();

}  // namespace b2cl
