// Translated CUDA kernels that fetch through textures.
// The paper's CUDA-to-OpenCL translation turns a texture reference
// into an image parameter plus a sampler parameter and tex1Dfetch / tex1D /
// tex2D / tex3D into read_imageX; these are the CUDA originals in that form,
// written against include/b2cl_device.cuh (whose tex* functions are the
// read built-ins) and launched through clSetKernelArg / clEnqueueNDRangeKernel
// with the image and sampler of b2clCreateTextureObject.
#include "b2cl_device.cuh"

// CUDA original:
// __global__ void fetch2d_f4(cudaTextureObject_t t, const float2* co, float4* out, int n) {
//   int i = blockIdx.x * blockDim.x + threadIdx.x;
//   if (i < n) out[i] = tex2D<float4>(t, co[i].x, co[i].y);
// }
extern "C" __global__ void fetch2d_f4(image2d_t t, sampler_t ts, const float2* co, float4* out, int n) {
  const int i = (int)get_global_id(0);
  if (i < n) out[i] = tex2D<float4>(t, ts, co[i].x, co[i].y);
}
extern "C" __global__ void fetch2d_f1(image2d_t t, sampler_t ts, const float2* co, float* out, int n) {
  const int i = (int)get_global_id(0);
  if (i < n) out[i] = tex2D<float>(t, ts, co[i].x, co[i].y);
}
// element-type reads of 8- and 16-bit integer textures
extern "C" __global__ void fetch2d_uc4(image2d_t t, sampler_t ts, const float2* co, uchar4* out, int n) {
  const int i = (int)get_global_id(0);
  if (i < n) out[i] = tex2D<uchar4>(t, ts, co[i].x, co[i].y);
}
extern "C" __global__ void fetch2d_s2(image2d_t t, sampler_t ts, const float2* co, short2* out, int n) {
  const int i = (int)get_global_id(0);
  if (i < n) out[i] = tex2D<short2>(t, ts, co[i].x, co[i].y);
}
extern "C" __global__ void fetch3d_f2(image3d_t t, sampler_t ts, const float4* co, float2* out, int n) {
  const int i = (int)get_global_id(0);
  if (i < n) out[i] = tex3D<float2>(t, ts, co[i].x, co[i].y, co[i].z);
}
extern "C" __global__ void fetch1d_f4(image1d_t t, sampler_t ts, const float* co, float4* out, int n) {
  const int i = (int)get_global_id(0);
  if (i < n) out[i] = tex1D<float4>(t, ts, co[i]);
}
// linear memory: tex1Dfetch(t, int) -- no sampler
extern "C" __global__ void fetch1dfetch_f4(image1d_buffer_t t, const int* xs, float4* out, int n) {
  const int i = (int)get_global_id(0);
  if (i < n) out[i] = tex1Dfetch<float4>(t, xs[i]);
}
// tex2DLayered(t, x, y, layer): co[i] = (x, y, layer, unused)
extern "C" __global__ void fetch2dlayered_f1(image2d_array_t t, sampler_t ts, const float4* co, float* out,
                                             int n) {
  const int i = (int)get_global_id(0);
  if (i < n) out[i] = tex2DLayered<float>(t, ts, co[i].x, co[i].y, (int)co[i].z);
}
