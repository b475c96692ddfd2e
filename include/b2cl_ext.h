/*
 * b2cl_ext.h -- b2cl extensions to the OpenCL subset of b2cl_cl.h.
 *
 * The paper runs read_imageX / write_imageX as device wrappers over the
 * CLImage pointer; there is no clBuildProgram in scope here
 * (the translator is out of scope), so the extensions below
 * expose those built-ins to the host as enqueue calls: one kernel launch
 * evaluates the built-in for every sample of a coordinate list or of an
 * affine output grid.  The per-sample arithmetic is [CL1.2 §8.1-8.3]
 * exactly as stated in b2cl_cl.h's header, with the readings of DESIGN.md
 * §3.  The remaining calls are runtime plumbing (torch streams and the torch
 * allocator, raw device pointers, CUDA IPC for the one-process-per-GPU
 * multi-device mode) and pure host validators that need no GPU.
 */
#ifndef B2CL_EXT_H
#define B2CL_EXT_H

#include "b2cl_cl.h"

#ifdef __cplusplus
extern "C" {
#endif

/* return class of the read / write built-in */
typedef cl_uint b2cl_rtype;
#define B2CL_RTYPE_FLOAT 0 /* read_imagef / write_imagef  (float4) */
#define B2CL_RTYPE_INT 1   /* read_imagei / write_imagei  (int4)   */
#define B2CL_RTYPE_UINT 2  /* read_imageui / write_imageui (uint4) */

/* coordinate element type of b2clEnqueueReadImageSamples */
typedef cl_uint b2cl_ctype;
#define B2CL_COORD_FLOAT 0
#define B2CL_COORD_INT 1

/* custom cl_mem_flags bit: allocate with cudaMalloc so that
 * b2clGetMemIpcHandle can export the object to another process. */
#define B2CL_MEM_IPC_EXPORTABLE ((cl_mem_flags)1 << 40)

/* custom cl_mem_flags bit for clCreateImage: TILED (block-linear) storage of a
 * CL_MEM_OBJECT_IMAGE2D -- 1 KiB tiles of 8 rows x 128 bytes (128 / elem_size
 * texels), tiles row-major (the north_star's "pitched and tiled image
 * storage").  The layout is internal and invisible through the API: every
 * pixel-box operation (Read/WriteImage, CopyImage with linear or tiled
 * partners, CopyImageToBuffer / BufferToImage, FillImage), the read / write
 * built-ins and translated kernels give the same texels as a pitched image;
 * clGetImageInfo reports CL_IMAGE_ROW_PITCH = width * elem_size (reading A46).
 * Any other image type, image shards, texture views and IPC import of a tiled
 * image -> CL_INVALID_VALUE. */
#define B2CL_MEM_TILED_IMAGE ((cl_mem_flags)1 << 41)

/* read_image{f,i,ui}(image, sampler, coord) for n coordinates
 * ([CL1.2 §6.12.14.2, §8.1-8.3]; steps a3-a7).
 *  coords:  buffer holding n coordinates starting at coords_offset, packed
 *           per sample as 1 (1D), 2 (2D) or 4 (3D; w ignored, reading A20)
 *           elements of 4 bytes: float (B2CL_COORD_FLOAT) or int32
 *           (B2CL_COORD_INT: requires an unnormalized, NEAREST sampler with a
 *           non-wrapping mode, reading A30).  coords_offset must be a
 *           multiple of the per-sample size.
 *  out:     n x 16 bytes (float4 / int4 / uint4) at out_offset (multiple of 16).
 * Errors: CL_INVALID_OPERATION if rtype does not match the channel type
 * (A7) or LINEAR is used with INT/UINT (A6); CL_INVALID_VALUE for a bad
 * offset / size; CL_INVALID_MEM_OBJECT / CL_INVALID_SAMPLER for bad handles.
 * n == 0 is a valid no-op. */
cl_int b2clEnqueueReadImageSamples(cl_command_queue command_queue, cl_mem image,
                                   cl_sampler sampler, b2cl_rtype rtype, b2cl_ctype ctype,
                                   cl_mem coords, size_t coords_offset, size_t num_samples,
                                   cl_mem out, size_t out_offset,
                                   cl_uint num_events_in_wait_list,
                                   const cl_event* event_wait_list, cl_event* event);

/* read_image{f,i,ui} over an output grid of out_dims[0] x out_dims[1] x
 * out_dims[2] samples, whose coordinates are an affine function of the
 * output index:  for k < image dims,
 *   coord[k] = ((affine[4k]*x + affine[4k+1]*y) + affine[4k+2]*z) + affine[4k+3]
 * with x,y,z converted to float and EVERY operation one fp32
 * round-to-nearest op in that order (no contraction, reading A2), so the
 * oracle reproduces the coordinates bit for bit.  The output is tightly
 * packed as [z][y][x][c], c < out_channels (1..4), 4 bytes per channel: the
 * first out_channels components of the result (e.g. 1 for CL_R images).
 * out_offset must be a multiple of 16. */
cl_int b2clEnqueueReadImageGrid(cl_command_queue command_queue, cl_mem image,
                                cl_sampler sampler, b2cl_rtype rtype, const float* affine,
                                const size_t* out_dims, cl_uint out_channels, cl_mem out,
                                size_t out_offset, cl_uint num_events_in_wait_list,
                                const cl_event* event_wait_list, cl_event* event);

/* The same over the output sub-box out_origin + [0, out_region): sample
 * (x,y,z) uses output indices (out_origin[0]+x, out_origin[1]+y,
 * out_origin[2]+z) in the affine map -- so a band of a larger output is
 * bit-identical to the same rows of the whole grid -- and is stored at
 * [z][y][x][c] of the region.  origin + region must stay below 2^31. */
cl_int b2clEnqueueReadImageGridRegion(cl_command_queue command_queue, cl_mem image,
                                      cl_sampler sampler, b2cl_rtype rtype, const float* affine,
                                      const size_t* out_origin, const size_t* out_region,
                                      cl_uint out_channels, cl_mem out, size_t out_offset,
                                      cl_uint num_events_in_wait_list,
                                      const cl_event* event_wait_list, cl_event* event);

/* An image SHARD: rows [begin, begin+count) (2D) or slices (3D) of a global
 * image described by global_desc, plus `halo` rows/slices on each side
 * (wrapping around the global extent), stored as a plain image of
 * count + 2*halo rows/slices: stored row s holds global row
 * (begin - halo + s) mod extent (row-sharded images).
 * The read built-ins (b2clEnqueueReadImage*) address the GLOBAL image --
 * global normalization, wrap and border -- and subtract the shard's first
 * stored row from the integer index only, so a shard reads bit-identically
 * to the whole image wherever its band + halo covers the filter footprint (a
 * tap outside it reads the nearest stored row; it is the caller's job to
 * provide the halo).  Every other operation (write_image, copies, fills,
 * Read/WriteImage, clGetImageInfo) addresses the stored rows as a plain
 * image.  count + 2*halo <= extent; 1D images cannot be sharded.
 * Errors as clCreateImage, and CL_INVALID_VALUE for a bad band. */
cl_mem b2clCreateImageShard(cl_context context, cl_mem_flags flags,
                            const cl_image_format* image_format,
                            const cl_image_desc* global_desc, size_t begin, size_t count,
                            size_t halo, void* host_ptr, cl_int* errcode_ret);

/* write_image{f,i,ui}(image, int coord, color) for n samples
 * ([CL1.2 §6.12.14.4, §8.3]; step a8).  int_coords: n x {1,2,4} int32 at
 * coords_offset; colors: n x 16 bytes at colors_offset (multiple of 16).
 * Out-of-range coordinates are no-ops (reading A15); if two samples hit the
 * same texel the surviving value is one of them (unspecified which). */
cl_int b2clEnqueueWriteImageSamples(cl_command_queue command_queue, cl_mem image,
                                    b2cl_rtype rtype, cl_mem int_coords, size_t coords_offset,
                                    size_t num_samples, cl_mem colors, size_t colors_offset,
                                    cl_uint num_events_in_wait_list,
                                    const cl_event* event_wait_list, cl_event* event);

/* ---- CUDA texture front end ----
 * The paper's CUDA-to-OpenCL direction translates a texture reference into
 * an image object and a sampler object added to the kernel's parameters, and
 * tex1Dfetch() / tex1D() / tex2D() / tex3D() into read_imageX().  A
 * b2cl_texture is that pair: b2clCreateTextureObject maps a CUDA-style
 * resource / texture description (the fields and enum values of CUDA's
 * cudaResourceDesc / cudaTextureDesc) onto an image VIEW of the resource's
 * storage (no copy: later writes to the storage are seen, as with a CUDA
 * texture) and a sampler; the device header's tex* functions
 * (b2cl_device.cuh) take the image and sampler and call the read built-ins.
 * Mapping (reading A40): wrap -> CLK_ADDRESS_REPEAT, clamp -> CLAMP_TO_EDGE,
 * mirror -> MIRRORED_REPEAT, border -> CLAMP (border 0 on the texture's
 * channels); point -> NEAREST, linear -> LINEAR; the channel type of the
 * view is the stored integer type for element-type reads and the matching
 * UNORM / SNORM type for normalized-float reads. */
#define B2CL_RESOURCE_ARRAY 0   /* an image (the translation of a cudaArray) */
#define B2CL_RESOURCE_LINEAR 2  /* linear memory in a buffer: tex1Dfetch only */
#define B2CL_RESOURCE_PITCH2D 3 /* pitched 2D memory in a buffer */
#define B2CL_CHANNEL_SIGNED 0   /* cudaChannelFormatKind */
#define B2CL_CHANNEL_UNSIGNED 1
#define B2CL_CHANNEL_FLOAT 2
#define B2CL_TEX_WRAP 0         /* cudaTextureAddressMode */
#define B2CL_TEX_CLAMP 1
#define B2CL_TEX_MIRROR 2
#define B2CL_TEX_BORDER 3
#define B2CL_TEX_POINT 0        /* cudaTextureFilterMode */
#define B2CL_TEX_LINEAR 1
#define B2CL_READ_ELEMENT_TYPE 0     /* cudaTextureReadMode */
#define B2CL_READ_NORMALIZED_FLOAT 1

/* cudaChannelFormatDesc: bits per channel x, y, z, w (1, 2 or 4 channels of
 * equal width: 8/16/32 for integers, 16/32 for floats) and their kind. */
typedef struct {
  cl_int x, y, z, w;
  cl_uint kind;
} b2cl_channel_format_desc;

typedef struct {
  cl_uint res_type;                /* B2CL_RESOURCE_* */
  cl_mem mem;                      /* ARRAY: an image (order R, RG or RGBA, not
                                      packed, not a shard); LINEAR / PITCH2D: a buffer */
  size_t offset;                   /* LINEAR / PITCH2D: byte offset into the buffer
                                      (a multiple of the texel size) */
  b2cl_channel_format_desc desc;   /* LINEAR / PITCH2D: the texel format */
  size_t size_in_bytes;            /* LINEAR: bytes of texels (a multiple of the texel size) */
  size_t width, height, pitch_in_bytes; /* PITCH2D (pitch: a multiple of the texel size) */
} b2cl_resource_desc;

typedef struct {
  cl_uint address_mode[3];  /* B2CL_TEX_WRAP..BORDER per axis; the sampled axes must agree */
  cl_uint filter_mode;      /* B2CL_TEX_POINT / LINEAR */
  cl_uint read_mode;        /* B2CL_READ_ELEMENT_TYPE / NORMALIZED_FLOAT */
  cl_int normalized_coords;
  float border_color[4];    /* must be 0 (OpenCL's border is fixed, reading A40) */
} b2cl_texture_desc;

typedef struct {
  cl_mem image;        /* the view (own reference) */
  cl_sampler sampler;  /* NULL for a LINEAR resource (tex1Dfetch takes none) */
  b2cl_rtype rtype;    /* read_imagef / i / ui of the view */
} b2cl_texture;

/* Creates the image view and sampler of a texture.  Errors:
 * CL_INVALID_CONTEXT / CL_INVALID_MEM_OBJECT for bad handles;
 * CL_IMAGE_FORMAT_NOT_SUPPORTED for a channel layout CUDA textures do not
 * have; CL_INVALID_VALUE for a bad resource (range, alignment), disagreeing
 * address modes on the sampled axes, wrap / mirror with unnormalized
 * coordinates, a normalized-float read of a 32-bit or float channel, or a
 * nonzero border colour; CL_INVALID_OPERATION for linear filtering of an
 * element-type integer read.  On error *tex is untouched. */
cl_int b2clCreateTextureObject(cl_context context, const b2cl_resource_desc* res_desc,
                               const b2cl_texture_desc* tex_desc, b2cl_texture* tex);
/* Releases the view and the sampler of *tex and clears it. */
cl_int b2clDestroyTextureObject(b2cl_texture* tex);

/* ---- runtime plumbing ---- */

/* A queue on an existing CUDA stream (e.g. torch.cuda.Stream.cuda_stream);
 * the stream is borrowed, not destroyed on release. */
cl_command_queue b2clCreateCommandQueueWithStream(cl_context context, cl_device_id device,
                                                  void* cuda_stream,
                                                  cl_command_queue_properties properties,
                                                  cl_int* errcode_ret);
/* The CUDA stream (cudaStream_t) a queue launches on. */
cl_int b2clGetCommandQueueStream(cl_command_queue command_queue, void** cuda_stream);
/* The CUDA device ordinal behind a cl_device_id. */
cl_int b2clGetDeviceOrdinal(cl_device_id device, cl_int* ordinal);

/* Device memory provider (e.g. torch.cuda.caching_allocator_alloc/delete).
 * alloc(size, device_ordinal, stream) returns a device pointer or NULL;
 * free(ptr, device_ordinal, stream).  Passing NULLs restores cudaMalloc /
 * cudaFree.  Affects objects created afterwards. */
typedef void* (*b2cl_alloc_fn)(size_t size, int device, void* stream);
typedef void (*b2cl_free_fn)(void* ptr, int device, void* stream);
cl_int b2clSetAllocator(b2cl_alloc_fn alloc_fn, b2cl_free_fn free_fn);

/* Wrap existing device memory (not owned, not freed) as a buffer resident
 * on `device` of `context`. */
cl_mem b2clCreateBufferFromDevicePointer(cl_context context, cl_device_id device,
                                         cl_mem_flags flags, void* device_ptr, size_t size,
                                         cl_int* errcode_ret);
/* Device pointer of a memory object on `device` (allocated on demand; no
 * migration).  For images this is the CLImage ptr (Fig. 6). */
cl_int b2clGetMemDevicePointer(cl_mem memobj, cl_device_id device, void** device_ptr);

/* CUDA IPC (the multi-device context across processes, one process per GPU;
 * SURVEY §8(e)).  b2clGetMemIpcHandle exports a buffer or image created with
 * B2CL_MEM_IPC_EXPORTABLE (its local cudaMalloc storage) as a 64-byte handle
 * (CL_INVALID_OPERATION otherwise).  The import calls open the handle on
 * `device` and return an object whose only valid copy is the EXPORTER's
 * memory (a peer GPU's, over NVLink), with the exporter's layout:
 *   - region copies and fills (clEnqueueCopyBuffer[Rect], CopyImage,
 *     CopyImageToBuffer, CopyBufferToImage, Fill*) read or write it in place,
 *     moving only the region over NVLink;
 *   - clEnqueueMigrateMemObjects, host transfers and the read built-ins first
 *     pull the whole content into a local store of the queue's device (one
 *     SM copy kernel reading the peer mapping), as in a multi-device context.
 * b2clCreateImageFromIpcHandle takes the exporter's cl_image_format and
 * cl_image_desc (no host pitches; the internal pitch is a function of them,
 * clGetImageInfo, reading A21) -- an image shard is imported as the plain
 * image of its stored rows.  Errors: CL_INVALID_CONTEXT / _DEVICE,
 * CL_INVALID_VALUE (NULL handle, host-pointer flags), the clCreateImage
 * format / descriptor codes, CL_OUT_OF_RESOURCES (the handle does not open).
 * The mapping is closed when the object is released (deferred like every
 * free, after the queues that used it are done). */
cl_int b2clGetMemIpcHandle(cl_mem memobj, void* handle64);
cl_mem b2clCreateBufferFromIpcHandle(cl_context context, cl_device_id device,
                                     const void* handle64, size_t size, cl_int* errcode_ret);
cl_mem b2clCreateImageFromIpcHandle(cl_context context, cl_device_id device, cl_mem_flags flags,
                                    const cl_image_format* image_format,
                                    const cl_image_desc* image_desc, const void* handle64,
                                    cl_int* errcode_ret);

/* clEnqueueCopyBuffer's semantics and validation ([CL1.2 §5.2.2]), moved by
 * the COPY ENGINES (cudaMemcpyAsync on the queue's stream, peer / IPC
 * pointers addressed in place) instead of the SM copy kernel: the reference
 * path the bench times beside the kernel for the NVLink roofline
 * (cudaMemcpyPeerAsync-class transfers). */
cl_int b2clEnqueueCopyBufferEngine(cl_command_queue command_queue, cl_mem src_buffer,
                                   cl_mem dst_buffer, size_t src_offset, size_t dst_offset,
                                   size_t size, cl_uint num_events_in_wait_list,
                                   const cl_event* event_wait_list, cl_event* event);
/* clEnqueueCopyBufferRect's semantics and validation ([CL1.2 §5.2.2]) on the
 * copy engines (cudaMemcpy3DAsync when both slice pitches are whole rows,
 * else cudaMemcpy2DAsync per slice): the SURVEY §8(d) config-4 reference. */
cl_int b2clEnqueueCopyBufferRectEngine(cl_command_queue command_queue, cl_mem src_buffer,
                                       cl_mem dst_buffer, const size_t* src_origin,
                                       const size_t* dst_origin, const size_t* region,
                                       size_t src_row_pitch, size_t src_slice_pitch,
                                       size_t dst_row_pitch, size_t dst_slice_pitch,
                                       cl_uint num_events_in_wait_list,
                                       const cl_event* event_wait_list, cl_event* event);
/* clEnqueueFillBuffer ([CL1.2 §5.2.3]) for pattern sizes 1, 2, 4 through
 * cuMemsetD8/D16/D32Async (the config-4 fill reference); other pattern sizes
 * -> CL_INVALID_VALUE. */
cl_int b2clEnqueueFillBufferEngine(cl_command_queue command_queue, cl_mem buffer, const void* pattern,
                                   size_t pattern_size, size_t offset, size_t size,
                                   cl_uint num_events_in_wait_list, const cl_event* event_wait_list,
                                   cl_event* event);

/* Number of b2cl kernels launched by this process so far (bench evidence). */
cl_ulong b2clGetKernelLaunchCount(void);

/* Name of the kernel the library's most recent launch from THIS host thread
 * used (e.g. "k_sample_grid_tile"): the enqueue calls pick one kernel family
 * per call (csrc/kernels/sample.cu launch_sample), and the bench reports which.
 * Returns a static NUL-terminated string owned by the library ("" before the
 * first launch); never NULL.  No side effects. */
const char* b2clGetLastKernelName(void);

/* ---- pure host validators (no GPU needed; the enqueue calls use them) ---- */

/* Errors of clEnqueueCopyBufferRect for buffers of src_size / dst_size
 * bytes (same_buffer != 0 when both are one object): CL_INVALID_VALUE,
 * CL_MEM_COPY_OVERLAP or CL_SUCCESS ([CL1.2 §5.2.2], reading A18). */
cl_int b2clValidateCopyBufferRect(size_t src_size, size_t dst_size, cl_int same_buffer,
                                  const size_t* src_origin, const size_t* dst_origin,
                                  const size_t* region, size_t src_row_pitch,
                                  size_t src_slice_pitch, size_t dst_row_pitch,
                                  size_t dst_slice_pitch);
/* Exact overlap test of two boxes with equal pitches in one buffer:
 * 1 if some byte is in both, else 0. */
cl_int b2clRectOverlap(const size_t* src_origin, const size_t* dst_origin, const size_t* region,
                       size_t row_pitch, size_t slice_pitch);
/* Errors of clEnqueueFillBuffer ([CL1.2 §5.2.3], reading A22). */
cl_int b2clValidateFillBuffer(size_t buffer_size, size_t pattern_size, size_t offset,
                              size_t size);
/* Errors of clCreateSampler (reading A5). */
cl_int b2clValidateSampler(cl_bool normalized_coords, cl_addressing_mode addressing_mode,
                           cl_filter_mode filter_mode);
/* Validates an image format / descriptor pair like clCreateImage (without
 * a host pointer) and returns the internal layout. */
cl_int b2clImageLayout(const cl_image_format* image_format, const cl_image_desc* image_desc,
                       size_t* elem_size, size_t* row_pitch, size_t* slice_pitch,
                       size_t* total_bytes);
/* The texture mapping of b2clCreateTextureObject: a texture description
 * over `sampled_dims` axes and the stored format of its resource (for an
 * ARRAY resource the image's format; otherwise the element-type format of
 * the channel description) -> the view's format, and the sampler's
 * normalized flag, addressing and filter mode, and the read's return class.
 * Same errors as b2clCreateTextureObject. */
cl_int b2clTextureMapping(const b2cl_texture_desc* tex_desc, cl_uint sampled_dims,
                          const cl_image_format* stored, cl_image_format* view,
                          cl_bool* normalized_coords, cl_addressing_mode* addressing_mode,
                          cl_filter_mode* filter_mode, b2cl_rtype* rtype);
/* The element-type image format of a cudaChannelFormatDesc (R / RG / RGBA of
 * SIGNED_INT*, UNSIGNED_INT*, HALF_FLOAT or FLOAT), or
 * CL_IMAGE_FORMAT_NOT_SUPPORTED. */
cl_int b2clChannelFormat(const b2cl_channel_format_desc* desc, cl_image_format* format);

/* Errors of an origin / region pixel box on an image of the given type and
 * size ([CL1.2 §5.3.3]). */
cl_int b2clValidateImageBox(cl_mem_object_type image_type, size_t width, size_t height,
                            size_t depth, const size_t* origin, const size_t* region);

#ifdef __cplusplus
}
#endif
#endif /* B2CL_EXT_H */
