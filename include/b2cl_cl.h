/*
 * b2cl_cl.h -- the OpenCL 1.2 host API subset exported by libb2cl.so.
 *
 * The paper re-implements each host API function of the source model as a
 * wrapper "that implements the same function" on the target (PAPER.md
 * P:97-99); handles are opaque pointers (cl_mem is
 * `struct _cl_mem*`) and image objects carry {ptr, size, format,
 * desc, row_pitch, slice_pitch, elem_size, channels} (Fig. 6).
 * So the Khronos names, prototypes and enum values ARE this interface; the
 * behaviour of each call is [CL1.2 §x] as cited per prototype, with the
 * readings listed in DESIGN.md §3 (A1..A33).  Values are restated from the
 * public Khronos cl.h (there is no CL/cl.h on the build box).
 *
 * Conventions for every entry point below:
 *  - Returns cl_int (CL_SUCCESS == 0, negative Khronos codes), or, for
 *    create calls, the handle (NULL on error) with *errcode_ret written when
 *    errcode_ret != NULL.
 *  - ALL argument validation happens before anything is enqueued: a call
 *    that returns an error has no side effect.
 *  - Handles start with reference count 1; clRetain* / clRelease* adjust it.
 *    A memory object's storage is freed when its count reaches 0, after the
 *    queues that used it have drained.
 *  - Host pointers passed to non-blocking reads/writes are owned by the
 *    caller and must stay valid until the returned event completes.
 *  - Every enqueue takes (num_events_in_wait_list, event_wait_list, event):
 *    the command waits for the listed events (cross-queue order is only the
 *    one events give, [CL1.2 §5.10]); if event != NULL a new event is
 *    returned (CUDA events underneath; profiling times when the queue was
 *    created with CL_QUEUE_PROFILING_ENABLE).
 *  - Commands execute on the GPU only; a CUDA failure maps to
 *    CL_OUT_OF_RESOURCES (launch/copy) or CL_MEM_OBJECT_ALLOCATION_FAILURE.
 */
#ifndef B2CL_CL_H
#define B2CL_CL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CL_API_CALL
#define CL_CALLBACK

typedef int8_t cl_char;
typedef uint8_t cl_uchar;
typedef int32_t cl_int;
typedef uint32_t cl_uint;
typedef int64_t cl_long;
typedef uint64_t cl_ulong;
typedef cl_uint cl_bool;
typedef cl_ulong cl_bitfield;
typedef cl_bitfield cl_device_type;
typedef cl_uint cl_platform_info;
typedef cl_uint cl_device_info;
typedef cl_bitfield cl_command_queue_properties;
typedef intptr_t cl_context_properties;
typedef cl_uint cl_context_info;
typedef cl_uint cl_command_queue_info;
typedef cl_uint cl_channel_order;
typedef cl_uint cl_channel_type;
typedef cl_bitfield cl_mem_flags;
typedef cl_uint cl_mem_object_type;
typedef cl_uint cl_mem_info;
typedef cl_bitfield cl_mem_migration_flags;
typedef cl_uint cl_image_info;
typedef cl_uint cl_addressing_mode;
typedef cl_uint cl_filter_mode;
typedef cl_uint cl_sampler_info;
typedef cl_uint cl_event_info;
typedef cl_uint cl_command_type;
typedef cl_uint cl_profiling_info;

typedef struct _cl_platform_id* cl_platform_id;
typedef struct _cl_device_id* cl_device_id;
typedef struct _cl_context* cl_context;
typedef struct _cl_command_queue* cl_command_queue;
typedef struct _cl_mem* cl_mem;
typedef struct _cl_sampler* cl_sampler;
typedef struct _cl_event* cl_event;
typedef struct _cl_program* cl_program;
typedef struct _cl_kernel* cl_kernel;
typedef cl_uint cl_program_build_info;
typedef cl_uint cl_kernel_info;

typedef struct _cl_image_format {
  cl_channel_order image_channel_order;
  cl_channel_type image_channel_data_type;
} cl_image_format;

typedef struct _cl_image_desc {
  cl_mem_object_type image_type;
  size_t image_width;
  size_t image_height;
  size_t image_depth;
  size_t image_array_size;
  size_t image_row_pitch;
  size_t image_slice_pitch;
  cl_uint num_mip_levels;
  cl_uint num_samples;
  cl_mem buffer;
} cl_image_desc;

/* ---- error codes ---- */
#define CL_SUCCESS 0
#define CL_DEVICE_NOT_FOUND -1
#define CL_DEVICE_NOT_AVAILABLE -2
#define CL_MEM_OBJECT_ALLOCATION_FAILURE -4
#define CL_OUT_OF_RESOURCES -5
#define CL_OUT_OF_HOST_MEMORY -6
#define CL_PROFILING_INFO_NOT_AVAILABLE -7
#define CL_MEM_COPY_OVERLAP -8
#define CL_IMAGE_FORMAT_MISMATCH -9
#define CL_IMAGE_FORMAT_NOT_SUPPORTED -10
#define CL_INVALID_VALUE -30
#define CL_INVALID_DEVICE_TYPE -31
#define CL_INVALID_PLATFORM -32
#define CL_INVALID_DEVICE -33
#define CL_INVALID_CONTEXT -34
#define CL_INVALID_QUEUE_PROPERTIES -35
#define CL_INVALID_COMMAND_QUEUE -36
#define CL_INVALID_HOST_PTR -37
#define CL_INVALID_MEM_OBJECT -38
#define CL_INVALID_IMAGE_FORMAT_DESCRIPTOR -39
#define CL_INVALID_IMAGE_SIZE -40
#define CL_INVALID_SAMPLER -41
#define CL_INVALID_EVENT_WAIT_LIST -57
#define CL_INVALID_EVENT -58
#define CL_INVALID_OPERATION -59
#define CL_INVALID_BUFFER_SIZE -61
#define CL_INVALID_IMAGE_DESCRIPTOR -65
#define CL_BUILD_PROGRAM_FAILURE -11
#define CL_INVALID_BINARY -42
#define CL_INVALID_BUILD_OPTIONS -43
#define CL_INVALID_PROGRAM -44
#define CL_INVALID_PROGRAM_EXECUTABLE -45
#define CL_INVALID_KERNEL_NAME -46
#define CL_INVALID_KERNEL -48
#define CL_INVALID_ARG_INDEX -49
#define CL_INVALID_ARG_VALUE -50
#define CL_INVALID_ARG_SIZE -51
#define CL_INVALID_KERNEL_ARGS -52
#define CL_INVALID_WORK_DIMENSION -53
#define CL_INVALID_WORK_GROUP_SIZE -54
#define CL_INVALID_WORK_ITEM_SIZE -55
#define CL_INVALID_GLOBAL_OFFSET -56
#define CL_PROGRAM_BUILD_STATUS 0x1181
#define CL_PROGRAM_BUILD_LOG 0x1183
#define CL_BUILD_SUCCESS 0
#define CL_BUILD_NONE -1
#define CL_BUILD_ERROR -2
#define CL_KERNEL_FUNCTION_NAME 0x1190
#define CL_KERNEL_NUM_ARGS 0x1191
#define CL_KERNEL_REFERENCE_COUNT 0x1192
#define CL_COMMAND_NDRANGE_KERNEL 0x11F0

#define CL_FALSE 0
#define CL_TRUE 1

/* ---- platform / device ---- */
#define CL_PLATFORM_PROFILE 0x0900
#define CL_PLATFORM_VERSION 0x0901
#define CL_PLATFORM_NAME 0x0902
#define CL_PLATFORM_VENDOR 0x0903
#define CL_PLATFORM_EXTENSIONS 0x0904

#define CL_DEVICE_TYPE_DEFAULT (1 << 0)
#define CL_DEVICE_TYPE_CPU (1 << 1)
#define CL_DEVICE_TYPE_GPU (1 << 2)
#define CL_DEVICE_TYPE_ACCELERATOR (1 << 3)
#define CL_DEVICE_TYPE_ALL 0xFFFFFFFF

#define CL_DEVICE_TYPE 0x1000
#define CL_DEVICE_VENDOR_ID 0x1001
#define CL_DEVICE_MAX_COMPUTE_UNITS 0x1002
#define CL_DEVICE_MAX_CLOCK_FREQUENCY 0x100C
#define CL_DEVICE_MAX_MEM_ALLOC_SIZE 0x1010
#define CL_DEVICE_IMAGE2D_MAX_WIDTH 0x1011
#define CL_DEVICE_IMAGE2D_MAX_HEIGHT 0x1012
#define CL_DEVICE_IMAGE3D_MAX_WIDTH 0x1013
#define CL_DEVICE_IMAGE3D_MAX_HEIGHT 0x1014
#define CL_DEVICE_IMAGE3D_MAX_DEPTH 0x1015
#define CL_DEVICE_IMAGE_SUPPORT 0x1016
#define CL_DEVICE_GLOBAL_MEM_SIZE 0x101F
#define CL_DEVICE_AVAILABLE 0x1027
#define CL_DEVICE_QUEUE_PROPERTIES 0x102A
#define CL_DEVICE_NAME 0x102B
#define CL_DEVICE_VENDOR 0x102C
#define CL_DRIVER_VERSION 0x102D
#define CL_DEVICE_PROFILE 0x102E
#define CL_DEVICE_VERSION 0x102F
#define CL_DEVICE_PLATFORM 0x1031
#define CL_DEVICE_IMAGE_MAX_BUFFER_SIZE 0x1040
#define CL_DEVICE_IMAGE_MAX_ARRAY_SIZE 0x1041

/* ---- context / queue ---- */
#define CL_CONTEXT_REFERENCE_COUNT 0x1080
#define CL_CONTEXT_DEVICES 0x1081
#define CL_CONTEXT_NUM_DEVICES 0x1083
#define CL_QUEUE_OUT_OF_ORDER_EXEC_MODE_ENABLE (1 << 0)
#define CL_QUEUE_PROFILING_ENABLE (1 << 1)
#define CL_QUEUE_CONTEXT 0x1090
#define CL_QUEUE_DEVICE 0x1091
#define CL_QUEUE_REFERENCE_COUNT 0x1092
#define CL_QUEUE_PROPERTIES 0x1093

/* ---- memory objects ---- */
#define CL_MEM_READ_WRITE (1 << 0)
#define CL_MEM_WRITE_ONLY (1 << 1)
#define CL_MEM_READ_ONLY (1 << 2)
#define CL_MEM_USE_HOST_PTR (1 << 3)
#define CL_MEM_ALLOC_HOST_PTR (1 << 4)
#define CL_MEM_COPY_HOST_PTR (1 << 5)
#define CL_MEM_HOST_WRITE_ONLY (1 << 7)
#define CL_MEM_HOST_READ_ONLY (1 << 8)
#define CL_MEM_HOST_NO_ACCESS (1 << 9)

#define CL_MIGRATE_MEM_OBJECT_HOST (1 << 0)
#define CL_MIGRATE_MEM_OBJECT_CONTENT_UNDEFINED (1 << 1)

#define CL_R 0x10B0
#define CL_A 0x10B1
#define CL_RG 0x10B2
#define CL_RA 0x10B3
#define CL_RGB 0x10B4
#define CL_RGBA 0x10B5
#define CL_BGRA 0x10B6
#define CL_ARGB 0x10B7
#define CL_INTENSITY 0x10B8
#define CL_LUMINANCE 0x10B9
#define CL_Rx 0x10BA
#define CL_RGx 0x10BB
#define CL_RGBx 0x10BC

#define CL_SNORM_INT8 0x10D0
#define CL_SNORM_INT16 0x10D1
#define CL_UNORM_INT8 0x10D2
#define CL_UNORM_INT16 0x10D3
#define CL_UNORM_SHORT_565 0x10D4
#define CL_UNORM_SHORT_555 0x10D5
#define CL_UNORM_INT_101010 0x10D6
#define CL_SIGNED_INT8 0x10D7
#define CL_SIGNED_INT16 0x10D8
#define CL_SIGNED_INT32 0x10D9
#define CL_UNSIGNED_INT8 0x10DA
#define CL_UNSIGNED_INT16 0x10DB
#define CL_UNSIGNED_INT32 0x10DC
#define CL_HALF_FLOAT 0x10DD
#define CL_FLOAT 0x10DE

#define CL_MEM_OBJECT_BUFFER 0x10F0
#define CL_MEM_OBJECT_IMAGE2D 0x10F1
#define CL_MEM_OBJECT_IMAGE3D 0x10F2
#define CL_MEM_OBJECT_IMAGE2D_ARRAY 0x10F3
#define CL_MEM_OBJECT_IMAGE1D 0x10F4
#define CL_MEM_OBJECT_IMAGE1D_ARRAY 0x10F5
#define CL_MEM_OBJECT_IMAGE1D_BUFFER 0x10F6

#define CL_MEM_TYPE 0x1100
#define CL_MEM_FLAGS 0x1101
#define CL_MEM_SIZE 0x1102
#define CL_MEM_HOST_PTR 0x1103
#define CL_MEM_MAP_COUNT 0x1104
#define CL_MEM_REFERENCE_COUNT 0x1105
#define CL_MEM_CONTEXT 0x1106
#define CL_MEM_ASSOCIATED_MEMOBJECT 0x1107
#define CL_MEM_OFFSET 0x1108

#define CL_IMAGE_FORMAT 0x1110
#define CL_IMAGE_ELEMENT_SIZE 0x1111
#define CL_IMAGE_ROW_PITCH 0x1112
#define CL_IMAGE_SLICE_PITCH 0x1113
#define CL_IMAGE_WIDTH 0x1114
#define CL_IMAGE_HEIGHT 0x1115
#define CL_IMAGE_DEPTH 0x1116
#define CL_IMAGE_ARRAY_SIZE 0x1117
#define CL_IMAGE_BUFFER 0x1118
#define CL_IMAGE_NUM_MIP_LEVELS 0x1119
#define CL_IMAGE_NUM_SAMPLES 0x111A

/* ---- samplers ---- */
#define CL_ADDRESS_NONE 0x1130
#define CL_ADDRESS_CLAMP_TO_EDGE 0x1131
#define CL_ADDRESS_CLAMP 0x1132
#define CL_ADDRESS_REPEAT 0x1133
#define CL_ADDRESS_MIRRORED_REPEAT 0x1134
#define CL_FILTER_NEAREST 0x1140
#define CL_FILTER_LINEAR 0x1141
#define CL_SAMPLER_REFERENCE_COUNT 0x1150
#define CL_SAMPLER_CONTEXT 0x1151
#define CL_SAMPLER_NORMALIZED_COORDS 0x1152
#define CL_SAMPLER_ADDRESSING_MODE 0x1153
#define CL_SAMPLER_FILTER_MODE 0x1154

/* ---- events ---- */
#define CL_EVENT_COMMAND_QUEUE 0x11D0
#define CL_EVENT_COMMAND_TYPE 0x11D1
#define CL_EVENT_REFERENCE_COUNT 0x11D2
#define CL_EVENT_COMMAND_EXECUTION_STATUS 0x11D3
#define CL_EVENT_CONTEXT 0x11D4
#define CL_COMPLETE 0x0
#define CL_RUNNING 0x1
#define CL_SUBMITTED 0x2
#define CL_QUEUED 0x3
#define CL_COMMAND_READ_BUFFER 0x11F3
#define CL_COMMAND_WRITE_BUFFER 0x11F4
#define CL_COMMAND_COPY_BUFFER 0x11F5
#define CL_COMMAND_READ_IMAGE 0x11F6
#define CL_COMMAND_WRITE_IMAGE 0x11F7
#define CL_COMMAND_COPY_IMAGE 0x11F8
#define CL_COMMAND_COPY_IMAGE_TO_BUFFER 0x11F9
#define CL_COMMAND_COPY_BUFFER_TO_IMAGE 0x11FA
#define CL_COMMAND_MARKER 0x11FE
#define CL_COMMAND_READ_BUFFER_RECT 0x1201
#define CL_COMMAND_WRITE_BUFFER_RECT 0x1202
#define CL_COMMAND_COPY_BUFFER_RECT 0x1203
#define CL_COMMAND_BARRIER 0x1205
#define CL_COMMAND_MIGRATE_MEM_OBJECTS 0x1206
#define CL_COMMAND_FILL_BUFFER 0x1207
#define CL_COMMAND_FILL_IMAGE 0x1208
#define CL_PROFILING_COMMAND_QUEUED 0x1280
#define CL_PROFILING_COMMAND_SUBMIT 0x1281
#define CL_PROFILING_COMMAND_START 0x1282
#define CL_PROFILING_COMMAND_END 0x1283

/* ================= platform, device, context, queue ================= */

/* [CL1.2 §4.1]  One platform ("b2cl") whose devices are the visible CUDA
 * devices of compute capability 10.0 (B200, sm_100a). */
cl_int CL_API_CALL clGetPlatformIDs(cl_uint num_entries, cl_platform_id* platforms,
                                    cl_uint* num_platforms);
cl_int CL_API_CALL clGetPlatformInfo(cl_platform_id platform, cl_platform_info param_name,
                                     size_t param_value_size, void* param_value,
                                     size_t* param_value_size_ret);
/* [CL1.2 §4.2]  CL_DEVICE_TYPE_GPU / DEFAULT / ALL list every device;
 * CPU / ACCELERATOR give CL_DEVICE_NOT_FOUND (no CPU device: no CPU fallback). */
cl_int CL_API_CALL clGetDeviceIDs(cl_platform_id platform, cl_device_type device_type,
                                  cl_uint num_entries, cl_device_id* devices,
                                  cl_uint* num_devices);
cl_int CL_API_CALL clGetDeviceInfo(cl_device_id device, cl_device_info param_name,
                                   size_t param_value_size, void* param_value,
                                   size_t* param_value_size_ret);

/* [CL1.2 §4.4]  A context over 1..N devices.  For N > 1 peer access is
 * enabled between every pair (NVLink / NVSwitch) and memory objects are made
 * resident per device on demand (see clEnqueueMigrateMemObjects).  The same
 * device may be listed twice (two queues on one GPU share its allocation). */
cl_context CL_API_CALL clCreateContext(const cl_context_properties* properties,
                                       cl_uint num_devices, const cl_device_id* devices,
                                       void(CL_CALLBACK* pfn_notify)(const char*, const void*,
                                                                     size_t, void*),
                                       void* user_data, cl_int* errcode_ret);
cl_int CL_API_CALL clRetainContext(cl_context context);
cl_int CL_API_CALL clReleaseContext(cl_context context);
cl_int CL_API_CALL clGetContextInfo(cl_context context, cl_context_info param_name,
                                    size_t param_value_size, void* param_value,
                                    size_t* param_value_size_ret);

/* [CL1.2 §5.1]  An in-order queue = one CUDA stream (non-blocking, owned).
 * CL_QUEUE_OUT_OF_ORDER_EXEC_MODE_ENABLE is accepted and executed in order
 * (a legal schedule).  CL_QUEUE_PROFILING_ENABLE records start/end events. */
cl_command_queue CL_API_CALL clCreateCommandQueue(cl_context context, cl_device_id device,
                                                  cl_command_queue_properties properties,
                                                  cl_int* errcode_ret);
cl_int CL_API_CALL clRetainCommandQueue(cl_command_queue command_queue);
cl_int CL_API_CALL clReleaseCommandQueue(cl_command_queue command_queue);
cl_int CL_API_CALL clGetCommandQueueInfo(cl_command_queue command_queue,
                                         cl_command_queue_info param_name,
                                         size_t param_value_size, void* param_value,
                                         size_t* param_value_size_ret);
cl_int CL_API_CALL clFlush(cl_command_queue command_queue);
/* blocks until every command in the queue has completed */
cl_int CL_API_CALL clFinish(cl_command_queue command_queue);

/* ================= memory objects and samplers ================= */

/* [CL1.2 §5.2.1]  Device allocation of `size` bytes (rounded up internally
 * to 256 B; CL_MEM_SIZE reports `size`).  CL_MEM_COPY_HOST_PTR uploads
 * host_ptr synchronously: the bytes are in device memory when the call
 * returns (visible to any queue's next command; host_ptr may be reused).
 * CL_MEM_USE_HOST_PTR -> CL_INVALID_VALUE
 * (reading A33); CL_MEM_ALLOC_HOST_PTR is accepted and ignored. */
cl_mem CL_API_CALL clCreateBuffer(cl_context context, cl_mem_flags flags, size_t size,
                                  void* host_ptr, cl_int* errcode_ret);

/* [CL1.2 §5.3.1]; the paper's CLImage (Fig. 6).
 * image_type: CL_MEM_OBJECT_IMAGE1D / IMAGE2D / IMAGE3D / IMAGE1D_ARRAY /
 * IMAGE2D_ARRAY / IMAGE1D_BUFFER.  An image array of L layers is stored as a
 * width x L (1D array) or width x height x L (2D array) image: layer l at
 * ptr + l*row_pitch (1D array) or ptr + l*slice_pitch (2D array); pixel boxes
 * select layers through origin/region[1] (1D array) or [2] (2D array), and
 * reads select the layer clamp(rint(coord), 0, L-1) ([CL1.2 §8.4]).  For a 1D
 * array image_slice_pitch is the host size of each layer (>= image_row_pitch,
 * 0 = image_row_pitch).  IMAGE1D_BUFFER: desc->buffer is a buffer of the same
 * context holding >= width*elem_size bytes; the image aliases its bytes
 * tightly packed (row_pitch = width*elem_size), retains it, and takes no
 * host_ptr, host pitches or host-pointer flags (CL_INVALID_VALUE, reading
 * A34); width <= CL_DEVICE_IMAGE_MAX_BUFFER_SIZE = 2^31-1 texels.  Formats: orders
 * R, A, RG, RA, RGBA with every non-packed channel type; BGRA and ARGB with
 * the 8-bit types; INTENSITY and LUMINANCE with UNORM/SNORM 8/16, HALF,
 * FLOAT ([CL1.2 §5.3.1.1]).  Storage is pitched linear in HBM: texel (i,j,k)
 * at ptr + k*slice_pitch + j*row_pitch + i*elem_size with
 * row_pitch = roundup(width*elem_size, 128) and slice_pitch =
 * row_pitch*height (reported by clGetImageInfo).  With
 * CL_MEM_COPY_HOST_PTR the contents are uploaded from host_ptr honouring
 * desc->image_row_pitch / image_slice_pitch (0 = tight), as the paper's
 * clCreateImage wrapper does with cudaMemcpy, complete when the call
 * returns (as clCreateBuffer). */
cl_mem CL_API_CALL clCreateImage(cl_context context, cl_mem_flags flags,
                                 const cl_image_format* image_format,
                                 const cl_image_desc* image_desc, void* host_ptr,
                                 cl_int* errcode_ret);
cl_int CL_API_CALL clGetSupportedImageFormats(cl_context context, cl_mem_flags flags,
                                              cl_mem_object_type image_type,
                                              cl_uint num_entries,
                                              cl_image_format* image_formats,
                                              cl_uint* num_image_formats);
cl_int CL_API_CALL clRetainMemObject(cl_mem memobj);
cl_int CL_API_CALL clReleaseMemObject(cl_mem memobj);
cl_int CL_API_CALL clGetMemObjectInfo(cl_mem memobj, cl_mem_info param_name,
                                      size_t param_value_size, void* param_value,
                                      size_t* param_value_size_ret);
/* [CL1.2 §5.3.7]: reports the Fig. 6 fields (format, elem_size, row_pitch,
 * slice_pitch, width, height, depth); SLICE_PITCH is 0 for 1D/2D images,
 * HEIGHT 0 for 1D, DEPTH 0 for 1D/2D. */
cl_int CL_API_CALL clGetImageInfo(cl_mem image, cl_image_info param_name,
                                  size_t param_value_size, void* param_value,
                                  size_t* param_value_size_ret);

/* [CL1.2 §5.5.1]  (normalized, addressing, filter).  REPEAT and
 * MIRRORED_REPEAT with unnormalized coordinates -> CL_INVALID_VALUE
 * (reading A5, stricter than the spec's "undefined"). */
cl_sampler CL_API_CALL clCreateSampler(cl_context context, cl_bool normalized_coords,
                                       cl_addressing_mode addressing_mode,
                                       cl_filter_mode filter_mode, cl_int* errcode_ret);
cl_int CL_API_CALL clRetainSampler(cl_sampler sampler);
cl_int CL_API_CALL clReleaseSampler(cl_sampler sampler);
cl_int CL_API_CALL clGetSamplerInfo(cl_sampler sampler, cl_sampler_info param_name,
                                    size_t param_value_size, void* param_value,
                                    size_t* param_value_size_ret);

/* ================= events ================= */
cl_int CL_API_CALL clWaitForEvents(cl_uint num_events, const cl_event* event_list);
cl_int CL_API_CALL clRetainEvent(cl_event event);
cl_int CL_API_CALL clReleaseEvent(cl_event event);
cl_int CL_API_CALL clGetEventInfo(cl_event event, cl_event_info param_name,
                                  size_t param_value_size, void* param_value,
                                  size_t* param_value_size_ret);
/* START/END in ns (relative to an arbitrary epoch, differences are exact to
 * the CUDA event resolution); needs CL_QUEUE_PROFILING_ENABLE. */
cl_int CL_API_CALL clGetEventProfilingInfo(cl_event event, cl_profiling_info param_name,
                                           size_t param_value_size, void* param_value,
                                           size_t* param_value_size_ret);
cl_int CL_API_CALL clEnqueueMarkerWithWaitList(cl_command_queue command_queue,
                                               cl_uint num_events_in_wait_list,
                                               const cl_event* event_wait_list,
                                               cl_event* event);
cl_int CL_API_CALL clEnqueueBarrierWithWaitList(cl_command_queue command_queue,
                                                cl_uint num_events_in_wait_list,
                                                const cl_event* event_wait_list,
                                                cl_event* event);

/* ================= bulk enqueues ================= */

/* [CL1.2 §5.2.2]  Host <-> buffer, contiguous.  blocking_* == CL_TRUE
 * returns after the copy completed. */
cl_int CL_API_CALL clEnqueueReadBuffer(cl_command_queue command_queue, cl_mem buffer,
                                       cl_bool blocking_read, size_t offset, size_t size,
                                       void* ptr, cl_uint num_events_in_wait_list,
                                       const cl_event* event_wait_list, cl_event* event);
cl_int CL_API_CALL clEnqueueWriteBuffer(cl_command_queue command_queue, cl_mem buffer,
                                        cl_bool blocking_write, size_t offset, size_t size,
                                        const void* ptr, cl_uint num_events_in_wait_list,
                                        const cl_event* event_wait_list, cl_event* event);

/* [CL1.2 §5.2.2] (step a10): the 3D byte box {region[0] bytes, region[1]
 * rows, region[2] slices} between a buffer (origin/pitches in bytes) and
 * host memory; pitch 0 -> region[0] / region[1]*row_pitch. */
cl_int CL_API_CALL clEnqueueReadBufferRect(cl_command_queue command_queue, cl_mem buffer,
                                           cl_bool blocking_read,
                                           const size_t* buffer_origin,
                                           const size_t* host_origin, const size_t* region,
                                           size_t buffer_row_pitch, size_t buffer_slice_pitch,
                                           size_t host_row_pitch, size_t host_slice_pitch,
                                           void* ptr, cl_uint num_events_in_wait_list,
                                           const cl_event* event_wait_list, cl_event* event);
cl_int CL_API_CALL clEnqueueWriteBufferRect(cl_command_queue command_queue, cl_mem buffer,
                                            cl_bool blocking_write,
                                            const size_t* buffer_origin,
                                            const size_t* host_origin, const size_t* region,
                                            size_t buffer_row_pitch, size_t buffer_slice_pitch,
                                            size_t host_row_pitch, size_t host_slice_pitch,
                                            const void* ptr, cl_uint num_events_in_wait_list,
                                            const cl_event* event_wait_list, cl_event* event);

/* [CL1.2 §5.2.2] contiguous device copy (a rect copy with one row). */
cl_int CL_API_CALL clEnqueueCopyBuffer(cl_command_queue command_queue, cl_mem src_buffer,
                                       cl_mem dst_buffer, size_t src_offset, size_t dst_offset,
                                       size_t size, cl_uint num_events_in_wait_list,
                                       const cl_event* event_wait_list, cl_event* event);

/* [CL1.2 §5.2.2] (step a9): for z < region[2], y < region[1]:
 *   dst[dst_off + z*dst_slice_pitch + y*dst_row_pitch + (0..region[0]-1)] =
 *   src[src_off + z*src_slice_pitch + y*src_row_pitch + (0..region[0]-1)],
 *   *_off = origin[2]*slice_pitch + origin[1]*row_pitch + origin[0].
 * Pitch 0 -> defaults.  Same buffer: pitches must be equal (reading A18)
 * and overlapping byte sets give CL_MEM_COPY_OVERLAP.  Runs the rect_copy
 * kernel (any alignment; 16-byte aligned stores, funnel-shifted loads). */
cl_int CL_API_CALL clEnqueueCopyBufferRect(cl_command_queue command_queue, cl_mem src_buffer,
                                           cl_mem dst_buffer, const size_t* src_origin,
                                           const size_t* dst_origin, const size_t* region,
                                           size_t src_row_pitch, size_t src_slice_pitch,
                                           size_t dst_row_pitch, size_t dst_slice_pitch,
                                           cl_uint num_events_in_wait_list,
                                           const cl_event* event_wait_list, cl_event* event);

/* [CL1.2 §5.2.3] (step a11): buf[offset + k] = pattern[k mod pattern_size]
 * for k < size; pattern_size in {1,2,4,...,128}, offset and size multiples
 * of it (reading A22).  The pattern is copied at enqueue time. */
cl_int CL_API_CALL clEnqueueFillBuffer(cl_command_queue command_queue, cl_mem buffer,
                                       const void* pattern, size_t pattern_size, size_t offset,
                                       size_t size, cl_uint num_events_in_wait_list,
                                       const cl_event* event_wait_list, cl_event* event);

/* [CL1.2 §5.3.3] (step a15): pixel box <-> host memory; origin/region in
 * pixels (2D: origin[2] = 0, region[2] = 1); host row_pitch /
 * slice_pitch in bytes, 0 = tight. */
cl_int CL_API_CALL clEnqueueReadImage(cl_command_queue command_queue, cl_mem image,
                                      cl_bool blocking_read, const size_t* origin,
                                      const size_t* region, size_t row_pitch, size_t slice_pitch,
                                      void* ptr, cl_uint num_events_in_wait_list,
                                      const cl_event* event_wait_list, cl_event* event);
cl_int CL_API_CALL clEnqueueWriteImage(cl_command_queue command_queue, cl_mem image,
                                       cl_bool blocking_write, const size_t* origin,
                                       const size_t* region, size_t input_row_pitch,
                                       size_t input_slice_pitch, const void* ptr,
                                       cl_uint num_events_in_wait_list,
                                       const cl_event* event_wait_list, cl_event* event);

/* [CL1.2 §5.3.3] (step a13): pixel box between two images of the same
 * format (else CL_IMAGE_FORMAT_MISMATCH); same image and overlapping boxes
 * -> CL_MEM_COPY_OVERLAP. */
cl_int CL_API_CALL clEnqueueCopyImage(cl_command_queue command_queue, cl_mem src_image,
                                      cl_mem dst_image, const size_t* src_origin,
                                      const size_t* dst_origin, const size_t* region,
                                      cl_uint num_events_in_wait_list,
                                      const cl_event* event_wait_list, cl_event* event);

/* [CL1.2 §5.3.4] (step a12): fill_color is float4, or int4 / uint4 for
 * SIGNED_INT* / UNSIGNED_INT* images (reading A23); it is converted once
 * with the write_image rules, on the device, and replicated over the box. */
cl_int CL_API_CALL clEnqueueFillImage(cl_command_queue command_queue, cl_mem image,
                                      const void* fill_color, const size_t* origin,
                                      const size_t* region, cl_uint num_events_in_wait_list,
                                      const cl_event* event_wait_list, cl_event* event);

/* [CL1.2 §5.3.5] (step a14): pixel box <-> tightly packed bytes
 * (region[0]*region[1]*region[2]*elem_size) at dst_offset / src_offset. */
cl_int CL_API_CALL clEnqueueCopyImageToBuffer(cl_command_queue command_queue, cl_mem src_image,
                                              cl_mem dst_buffer, const size_t* src_origin,
                                              const size_t* region, size_t dst_offset,
                                              cl_uint num_events_in_wait_list,
                                              const cl_event* event_wait_list,
                                              cl_event* event);
cl_int CL_API_CALL clEnqueueCopyBufferToImage(cl_command_queue command_queue, cl_mem src_buffer,
                                              cl_mem dst_image, size_t src_offset,
                                              const size_t* dst_origin, const size_t* region,
                                              cl_uint num_events_in_wait_list,
                                              const cl_event* event_wait_list,
                                              cl_event* event);

/* [CL1.2 §5.4.4] (step a16): make each object's valid copy resident on the
 * queue's device: a device-to-device pull over NVLink (SM copy kernel on
 * peer memory) from a device holding a valid copy.  CONTENT_UNDEFINED: no
 * copy, ownership only.  HOST: the content is kept valid on its current
 * device (device memory is the only storage; reading A24). */
cl_int CL_API_CALL clEnqueueMigrateMemObjects(cl_command_queue command_queue,
                                              cl_uint num_mem_objects, const cl_mem* mem_objects,
                                              cl_mem_migration_flags flags,
                                              cl_uint num_events_in_wait_list,
                                              const cl_event* event_wait_list, cl_event* event);

/* ================= programs and kernels (launch glue) ================= */

/* The paper builds an OpenCL program by translating it to CUDA C, compiling
 * it with nvcc and loading the module with cuModuleLoad.  Here the
 * translated kernel (written against include/b2cl_device.cuh) is compiled
 * with nvcc ahead of time, and its cubin / fatbin / PTX image is the program
 * binary.  binaries[i] (lengths[i] bytes) is the module for devices[i];
 * binary_status[i] receives CL_SUCCESS or CL_INVALID_BINARY. */
cl_program CL_API_CALL clCreateProgramWithBinary(cl_context context, cl_uint num_devices,
                                                 const cl_device_id* device_list,
                                                 const size_t* lengths,
                                                 const unsigned char** binaries,
                                                 cl_int* binary_status, cl_int* errcode_ret);
/* Loads the module on every device of the program (cudaLibraryLoadData);
 * options are ignored; CL_BUILD_PROGRAM_FAILURE if a device rejects it. */
cl_int CL_API_CALL clBuildProgram(cl_program program, cl_uint num_devices,
                                  const cl_device_id* device_list, const char* options,
                                  void(CL_CALLBACK* pfn_notify)(cl_program, void*),
                                  void* user_data);
cl_int CL_API_CALL clGetProgramBuildInfo(cl_program program, cl_device_id device,
                                         cl_program_build_info param_name,
                                         size_t param_value_size, void* param_value,
                                         size_t* param_value_size_ret);
cl_int CL_API_CALL clRetainProgram(cl_program program);
cl_int CL_API_CALL clReleaseProgram(cl_program program);

/* A __global__ function of the built program (extern "C" name). */
cl_kernel CL_API_CALL clCreateKernel(cl_program program, const char* kernel_name,
                                     cl_int* errcode_ret);
cl_int CL_API_CALL clRetainKernel(cl_kernel kernel);
cl_int CL_API_CALL clReleaseKernel(cl_kernel kernel);
cl_int CL_API_CALL clGetKernelInfo(cl_kernel kernel, cl_kernel_info param_name,
                                   size_t param_value_size, void* param_value,
                                   size_t* param_value_size_ret);

/* Records argument arg_index, as the paper's wrapper does ("the parameters
 * of cuLaunchKernel() ... are collected when clSetKernelArg() is called",
 * P:139).  arg_value == NULL: a __local argument of arg_size bytes -- the
 * kernel receives the size (size_t) and the launch reserves the sum of all
 * __local sizes as dynamic shared memory (Fig. 5(b)).  arg_value
 * pointing to a cl_mem: a buffer passes its device pointer, an image its
 * descriptor by value (b2cl_device.cuh image*_t).  To a cl_sampler: its
 * 32-bit CLK_* bits.  Anything else: the arg_size bytes. */
cl_int CL_API_CALL clSetKernelArg(cl_kernel kernel, cl_uint arg_index, size_t arg_size,
                                  const void* arg_value);

/* [CL1.2 §5.8]: work_dim 1..3, global_work_size[d] > 0, local_work_size
 * (or a chosen one when NULL) must divide it (CL_INVALID_WORK_GROUP_SIZE)
 * with at most 1024 work-items per group; global_work_offset is passed to
 * get_global_id through the module's __b2cl_global_offset.  One
 * cudaLaunchKernel: grid = global / local, block = local.  Buffers and
 * images passed to the kernel count as written by it (residency). */
cl_int CL_API_CALL clEnqueueNDRangeKernel(cl_command_queue command_queue, cl_kernel kernel,
                                          cl_uint work_dim, const size_t* global_work_offset,
                                          const size_t* global_work_size,
                                          const size_t* local_work_size,
                                          cl_uint num_events_in_wait_list,
                                          const cl_event* event_wait_list, cl_event* event);

#ifdef __cplusplus
}
#endif
#endif /* B2CL_CL_H */
