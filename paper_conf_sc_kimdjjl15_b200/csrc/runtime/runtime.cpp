// runtime.cpp -- the OpenCL 1.2 host API subset of libb2cl, over the CUDA
// runtime (the paper's wrapper runtime, P:97-99, P:119, P:139, P:426-428,
// re-designed for B200: one CUDA stream per queue, pitched images in HBM,
// memory objects per context with per-device residency, peer pulls over
// NVLink for cross-device migration).
//
// Every enqueue: (1) validates all arguments (no side effect on error),
// (2) makes the touched objects resident on the queue's device,
// (3) waits for the wait-list events, (4) launches ONE kernel (or a copy
// engine transfer for host memory), (5) returns an event if asked.
#include <cuda.h>
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <atomic>
#include <functional>
#include <mutex>
#include <new>
#include <set>
#include <string>
#include <vector>

#include "../kernels/launch.h"
#include "internal.h"

using namespace b2cl;

// ===================================================================== objects
struct _cl_platform_id {
  int magic;
};

struct _cl_device_id {
  int ordinal;
  cudaDeviceProp prop;
};

struct _cl_context {
  std::atomic<int> ref{1};
  std::vector<cl_device_id> devs;  // as given (may repeat a device)
  std::vector<int> ordinals;       // distinct CUDA ordinals
  bool peer[64][64] = {};          // peer access enabled (dst row, src col)
};

struct _cl_command_queue {
  std::atomic<int> ref{1};
  cl_context ctx;
  cl_device_id dev;
  cudaStream_t stream;
  bool owns_stream;
  cl_command_queue_properties props;
};

struct Store {
  int ordinal = -1;     // the CUDA device whose address space holds ptr
  char* ptr = nullptr;
  int kind = 0;  // 0 none, 1 cudaMalloc, 2 allocator hook, 3 borrowed, 4 IPC import
};

// An IPC-imported store (kind 4) is ANOTHER process's memory -- a peer GPU's
// over NVLink, or a region of this GPU owned by another process -- mapped into
// `ordinal`'s address space.  It is not this device's local copy: its valid
// bit is kRemoteBit, so clEnqueueMigrateMemObjects (or a sampling read) pulls
// it into a local store, while region copies read / write it in place.
constexpr int kRemoteBit = 63;
static int bit_of(const Store& s) { return s.kind == 4 ? kRemoteBit : s.ordinal; }

struct _cl_mem {
  std::atomic<int> ref{1};
  cl_context ctx;
  cl_mem_object_type type;
  cl_mem_flags flags;
  size_t size = 0;        // CL_MEM_SIZE (user size; images: total bytes)
  size_t alloc_size = 0;  // rounded to 256 B
  ImageLayout img{};      // images only (a shard: the layout of its stored rows)
  // image shards (b2clCreateImageShard): the outer axis (2D rows / 3D slices)
  // of a global image of extent shard_extent; stored row s is global index
  // (shard_ob + s) mod shard_extent
  bool shard = false;
  size_t shard_extent = 0;
  long long shard_ob = 0;
  cl_image_format fmt{};
  cl_image_desc desc{};
  // a 1D image buffer (CL_MEM_OBJECT_IMAGE1D_BUFFER) or a texture's image
  // view owns no storage: its texels are the bytes of this object (a buffer
  // or an image) from byte parent_off on, and it retains the object
  cl_mem parent = nullptr;
  size_t parent_off = 0;
  std::mutex mu;
  std::vector<Store> stores;
  uint64_t valid = 0;                   // bit per ordinal holding valid content
  std::set<cl_command_queue> users;     // queues that enqueued work on it
};

struct _cl_sampler {
  std::atomic<int> ref{1};
  cl_context ctx;
  cl_bool norm;
  cl_addressing_mode addr;
  cl_filter_mode filt;
};

struct _cl_event {
  std::atomic<int> ref{1};
  cl_context ctx;
  cl_command_queue queue;
  cl_command_type type;
  int ordinal;
  cudaEvent_t start = nullptr, end = nullptr;
};

// ===================================================================== globals
static _cl_platform_id g_platform{0x62326c};
static std::vector<_cl_device_id> g_devices;
static std::once_flag g_dev_once;
static std::mutex g_mu;                       // guards the registries below
static std::set<cl_command_queue> g_queues;   // live queues
static std::set<cl_mem> g_mems;
static std::set<cl_context> g_contexts;
static std::set<cl_sampler> g_samplers;
static std::set<cl_event> g_events;
static b2cl_alloc_fn g_alloc = nullptr;
static b2cl_free_fn g_free = nullptr;
static cudaEvent_t g_epoch[64] = {};

static void init_devices() {
  std::call_once(g_dev_once, [] {
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess) {
      cudaGetLastError();
      n = 0;
    }
    for (int i = 0; i < n; ++i) {
      _cl_device_id d;
      d.ordinal = i;
      if (cudaGetDeviceProperties(&d.prop, i) != cudaSuccess) continue;
      if (d.prop.major != 10 || d.prop.minor != 0) continue;  // kernels are sm_100a only
      g_devices.push_back(d);
    }
  });
}

template <class T>
static bool live(const std::set<T>& reg, T h) {
  std::lock_guard<std::mutex> g(g_mu);
  return h && reg.count(h);
}

// Retain / release under the registry lock: the liveness check and the count
// change are one step, so two threads releasing the last reference cannot
// both destroy the object, and a release racing a retain never resurrects a
// destroyed one.  release_ref returns -1 (not live), 0 (still referenced) or 1
// (last reference: already removed from the registry, the caller destroys).
template <class T>
static bool retain_ref(std::set<T>& reg, T h) {
  std::lock_guard<std::mutex> g(g_mu);
  if (!h || !reg.count(h)) return false;
  h->ref++;
  return true;
}
template <class T>
static int release_ref(std::set<T>& reg, T h) {
  std::lock_guard<std::mutex> g(g_mu);
  if (!h || !reg.count(h)) return -1;
  if (--h->ref > 0) return 0;
  reg.erase(h);
  return 1;
}

static cl_int cuda_err(cudaError_t e) {
  if (e == cudaSuccess) return CL_SUCCESS;
  cudaGetLastError();
  return e == cudaErrorMemoryAllocation ? CL_MEM_OBJECT_ALLOCATION_FAILURE : CL_OUT_OF_RESOURCES;
}

// current-device guard: the runtime sets the queue's device for its calls and
// restores the caller's (torch's) device afterwards.
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int ordinal) {
    cudaGetDevice(&prev);
    if (prev != ordinal) cudaSetDevice(ordinal);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

template <class T>
static cl_int get_info(const T& v, size_t size, void* out, size_t* size_ret) {
  if (size_ret) *size_ret = sizeof(T);
  if (out) {
    if (size < sizeof(T)) return CL_INVALID_VALUE;
    memcpy(out, &v, sizeof(T));
  }
  return CL_SUCCESS;
}
static cl_int get_str(const char* s, size_t size, void* out, size_t* size_ret) {
  const size_t n = strlen(s) + 1;
  if (size_ret) *size_ret = n;
  if (out) {
    if (size < n) return CL_INVALID_VALUE;
    memcpy(out, s, n);
  }
  return CL_SUCCESS;
}

#define SET_ERR(e)             \
  do {                         \
    if (errcode_ret) *errcode_ret = (e); \
  } while (0)

// ===================================================================== platform / device
extern "C" cl_int clGetPlatformIDs(cl_uint num_entries, cl_platform_id* platforms,
                                   cl_uint* num_platforms) {
  if ((num_entries == 0 && platforms) || (!platforms && !num_platforms)) return CL_INVALID_VALUE;
  if (platforms && num_entries > 0) platforms[0] = &g_platform;
  if (num_platforms) *num_platforms = 1;
  return CL_SUCCESS;
}

extern "C" cl_int clGetPlatformInfo(cl_platform_id platform, cl_platform_info name, size_t size,
                                    void* value, size_t* size_ret) {
  if (platform && platform != &g_platform) return CL_INVALID_PLATFORM;
  switch (name) {
    case CL_PLATFORM_PROFILE: return get_str("FULL_PROFILE", size, value, size_ret);
    case CL_PLATFORM_VERSION: return get_str("OpenCL 1.2 b2cl (B200 sm_100a)", size, value, size_ret);
    case CL_PLATFORM_NAME: return get_str("b2cl", size, value, size_ret);
    case CL_PLATFORM_VENDOR: return get_str("b2cl", size, value, size_ret);
    case CL_PLATFORM_EXTENSIONS: return get_str("", size, value, size_ret);
    default: return CL_INVALID_VALUE;
  }
}

static bool valid_device(cl_device_id d) {
  init_devices();
  for (auto& x : g_devices)
    if (&x == d) return true;
  return false;
}

extern "C" cl_int clGetDeviceIDs(cl_platform_id platform, cl_device_type type, cl_uint num_entries,
                                 cl_device_id* devices, cl_uint* num_devices) {
  if (platform && platform != &g_platform) return CL_INVALID_PLATFORM;
  if ((num_entries == 0 && devices) || (!devices && !num_devices)) return CL_INVALID_VALUE;
  const cl_device_type known = CL_DEVICE_TYPE_DEFAULT | CL_DEVICE_TYPE_CPU | CL_DEVICE_TYPE_GPU |
                               CL_DEVICE_TYPE_ACCELERATOR;
  if (type != CL_DEVICE_TYPE_ALL && (type & ~known)) return CL_INVALID_DEVICE_TYPE;
  init_devices();
  const bool gpu = type == CL_DEVICE_TYPE_ALL || (type & (CL_DEVICE_TYPE_GPU | CL_DEVICE_TYPE_DEFAULT));
  const cl_uint n = gpu ? (cl_uint)g_devices.size() : 0;
  if (n == 0) return CL_DEVICE_NOT_FOUND;
  if (devices)
    for (cl_uint i = 0; i < std::min(n, num_entries); ++i) devices[i] = &g_devices[i];
  if (num_devices) *num_devices = n;
  return CL_SUCCESS;
}

extern "C" cl_int clGetDeviceInfo(cl_device_id d, cl_device_info name, size_t size, void* value,
                                  size_t* size_ret) {
  if (!valid_device(d)) return CL_INVALID_DEVICE;
  const cudaDeviceProp& p = d->prop;
  switch (name) {
    case CL_DEVICE_TYPE: return get_info<cl_device_type>(CL_DEVICE_TYPE_GPU, size, value, size_ret);
    case CL_DEVICE_VENDOR_ID: return get_info<cl_uint>(0x10DE, size, value, size_ret);
    case CL_DEVICE_MAX_COMPUTE_UNITS: return get_info<cl_uint>(p.multiProcessorCount, size, value, size_ret);
    case CL_DEVICE_MAX_CLOCK_FREQUENCY: {
      int khz = 0;
      cudaDeviceGetAttribute(&khz, cudaDevAttrClockRate, d->ordinal);
      return get_info<cl_uint>(khz / 1000, size, value, size_ret);
    }
    case CL_DEVICE_GLOBAL_MEM_SIZE: return get_info<cl_ulong>(p.totalGlobalMem, size, value, size_ret);
    case CL_DEVICE_MAX_MEM_ALLOC_SIZE: return get_info<cl_ulong>(p.totalGlobalMem, size, value, size_ret);
    case CL_DEVICE_IMAGE_SUPPORT: return get_info<cl_bool>(CL_TRUE, size, value, size_ret);
    case CL_DEVICE_IMAGE2D_MAX_WIDTH:
    case CL_DEVICE_IMAGE2D_MAX_HEIGHT: return get_info<size_t>(kMax2D, size, value, size_ret);
    case CL_DEVICE_IMAGE3D_MAX_WIDTH:
    case CL_DEVICE_IMAGE3D_MAX_HEIGHT:
    case CL_DEVICE_IMAGE3D_MAX_DEPTH: return get_info<size_t>(kMax3D, size, value, size_ret);
    case CL_DEVICE_IMAGE_MAX_BUFFER_SIZE: return get_info<size_t>(kMaxBuffer, size, value, size_ret);
    case CL_DEVICE_IMAGE_MAX_ARRAY_SIZE: return get_info<size_t>(kMaxArray, size, value, size_ret);
    case CL_DEVICE_AVAILABLE: return get_info<cl_bool>(CL_TRUE, size, value, size_ret);
    case CL_DEVICE_QUEUE_PROPERTIES:
      return get_info<cl_command_queue_properties>(
          CL_QUEUE_PROFILING_ENABLE | CL_QUEUE_OUT_OF_ORDER_EXEC_MODE_ENABLE, size, value, size_ret);
    case CL_DEVICE_NAME: return get_str(p.name, size, value, size_ret);
    case CL_DEVICE_VENDOR: return get_str("NVIDIA Corporation", size, value, size_ret);
    case CL_DRIVER_VERSION: return get_str("b2cl 0.1", size, value, size_ret);
    case CL_DEVICE_PROFILE: return get_str("FULL_PROFILE", size, value, size_ret);
    case CL_DEVICE_VERSION: return get_str("OpenCL 1.2 b2cl", size, value, size_ret);
    case CL_DEVICE_PLATFORM: return get_info<cl_platform_id>(&g_platform, size, value, size_ret);
    default: return CL_INVALID_VALUE;
  }
}

extern "C" cl_int b2clGetDeviceOrdinal(cl_device_id d, cl_int* ordinal) {
  if (!valid_device(d)) return CL_INVALID_DEVICE;
  if (!ordinal) return CL_INVALID_VALUE;
  *ordinal = d->ordinal;
  return CL_SUCCESS;
}

// ===================================================================== context
extern "C" cl_context clCreateContext(const cl_context_properties* props, cl_uint num_devices,
                                      const cl_device_id* devices,
                                      void(CL_CALLBACK* notify)(const char*, const void*, size_t, void*),
                                      void* user_data, cl_int* errcode_ret) {
  (void)user_data;
  if (num_devices == 0 || !devices) { SET_ERR(CL_INVALID_VALUE); return nullptr; }
  if (!notify && user_data) { SET_ERR(CL_INVALID_VALUE); return nullptr; }
  if (props) {
    for (const cl_context_properties* p = props; *p; p += 2) {
      if (*p != 0x1084 /* CL_CONTEXT_PLATFORM */ ||
          reinterpret_cast<cl_platform_id>(p[1]) != &g_platform) {
        SET_ERR(CL_INVALID_PLATFORM);
        return nullptr;
      }
    }
  }
  for (cl_uint i = 0; i < num_devices; ++i)
    if (!valid_device(devices[i])) { SET_ERR(CL_INVALID_DEVICE); return nullptr; }
  auto* c = new (std::nothrow) _cl_context();
  if (!c) { SET_ERR(CL_OUT_OF_HOST_MEMORY); return nullptr; }
  for (cl_uint i = 0; i < num_devices; ++i) {
    c->devs.push_back(devices[i]);
    if (std::find(c->ordinals.begin(), c->ordinals.end(), devices[i]->ordinal) == c->ordinals.end())
      c->ordinals.push_back(devices[i]->ordinal);
  }
  // all-pairs peer access over NVLink / NVSwitch
  for (int a : c->ordinals) {
    DeviceGuard g(a);
    if (!g_epoch[a]) cudaEventCreate(&g_epoch[a]), cudaEventRecord(g_epoch[a], 0);
    for (int b : c->ordinals) {
      if (a == b) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, a, b);
      if (can) {
        cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
        if (e == cudaSuccess || e == cudaErrorPeerAccessAlreadyEnabled) c->peer[a][b] = true;
        cudaGetLastError();
      }
    }
  }
  {
    std::lock_guard<std::mutex> g(g_mu);
    g_contexts.insert(c);
  }
  SET_ERR(CL_SUCCESS);
  return c;
}

static void reap_frees(bool block);

extern "C" cl_int clRetainContext(cl_context c) {
  return retain_ref(g_contexts, c) ? CL_SUCCESS : CL_INVALID_CONTEXT;
}

extern "C" cl_int clReleaseContext(cl_context c) {
  const int r = release_ref(g_contexts, c);
  if (r < 0) return CL_INVALID_CONTEXT;
  if (r == 1) {
    reap_frees(true);  // the context's last memory objects' deferred frees
    delete c;
  }
  return CL_SUCCESS;
}

extern "C" cl_int clGetContextInfo(cl_context c, cl_context_info name, size_t size, void* value,
                                   size_t* size_ret) {
  if (!live(g_contexts, c)) return CL_INVALID_CONTEXT;
  switch (name) {
    case CL_CONTEXT_REFERENCE_COUNT: return get_info<cl_uint>(c->ref.load(), size, value, size_ret);
    case CL_CONTEXT_NUM_DEVICES: return get_info<cl_uint>((cl_uint)c->devs.size(), size, value, size_ret);
    case CL_CONTEXT_DEVICES: {
      const size_t n = c->devs.size() * sizeof(cl_device_id);
      if (size_ret) *size_ret = n;
      if (value) {
        if (size < n) return CL_INVALID_VALUE;
        memcpy(value, c->devs.data(), n);
      }
      return CL_SUCCESS;
    }
    default: return CL_INVALID_VALUE;
  }
}

static bool ctx_has_device(cl_context c, cl_device_id d) {
  return std::find(c->devs.begin(), c->devs.end(), d) != c->devs.end();
}

// ===================================================================== queue
static cl_command_queue make_queue(cl_context c, cl_device_id d, cl_command_queue_properties props,
                                   void* stream, cl_int* errcode_ret) {
  if (!live(g_contexts, c)) { SET_ERR(CL_INVALID_CONTEXT); return nullptr; }
  if (!valid_device(d) || !ctx_has_device(c, d)) { SET_ERR(CL_INVALID_DEVICE); return nullptr; }
  if (props & ~(cl_command_queue_properties)(CL_QUEUE_PROFILING_ENABLE |
                                             CL_QUEUE_OUT_OF_ORDER_EXEC_MODE_ENABLE)) {
    SET_ERR(CL_INVALID_VALUE);
    return nullptr;
  }
  auto* q = new (std::nothrow) _cl_command_queue();
  if (!q) { SET_ERR(CL_OUT_OF_HOST_MEMORY); return nullptr; }
  q->ctx = c;
  q->dev = d;
  q->props = props;
  if (stream) {
    q->stream = static_cast<cudaStream_t>(stream);
    q->owns_stream = false;
  } else {
    DeviceGuard g(d->ordinal);
    cudaError_t e = cudaStreamCreateWithFlags(&q->stream, cudaStreamNonBlocking);
    if (e != cudaSuccess) {
      delete q;
      SET_ERR(cuda_err(e));
      return nullptr;
    }
    q->owns_stream = true;
  }
  c->ref++;
  {
    std::lock_guard<std::mutex> g(g_mu);
    g_queues.insert(q);
  }
  SET_ERR(CL_SUCCESS);
  return q;
}

extern "C" cl_command_queue clCreateCommandQueue(cl_context c, cl_device_id d,
                                                 cl_command_queue_properties props,
                                                 cl_int* errcode_ret) {
  return make_queue(c, d, props, nullptr, errcode_ret);
}

extern "C" cl_command_queue b2clCreateCommandQueueWithStream(cl_context c, cl_device_id d,
                                                             void* stream,
                                                             cl_command_queue_properties props,
                                                             cl_int* errcode_ret) {
  return make_queue(c, d, props, stream, errcode_ret);
}

extern "C" cl_int b2clGetCommandQueueStream(cl_command_queue q, void** stream) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  if (!stream) return CL_INVALID_VALUE;
  *stream = q->stream;
  return CL_SUCCESS;
}

extern "C" cl_int clRetainCommandQueue(cl_command_queue q) {
  return retain_ref(g_queues, q) ? CL_SUCCESS : CL_INVALID_COMMAND_QUEUE;
}

extern "C" cl_int clReleaseCommandQueue(cl_command_queue q) {
  const int r = release_ref(g_queues, q);
  if (r < 0) return CL_INVALID_COMMAND_QUEUE;
  if (r == 1) {
    {
      DeviceGuard g(q->dev->ordinal);
      cudaStreamSynchronize(q->stream);  // implicit flush + finish before teardown
      if (q->owns_stream) cudaStreamDestroy(q->stream);
    }
    {
      std::lock_guard<std::mutex> g(g_mu);
      for (cl_mem m : g_mems) {
        std::lock_guard<std::mutex> gm(m->mu);
        m->users.erase(q);
      }
    }
    reap_frees(false);
    cl_context c = q->ctx;
    delete q;
    clReleaseContext(c);
  }
  return CL_SUCCESS;
}

extern "C" cl_int clGetCommandQueueInfo(cl_command_queue q, cl_command_queue_info name,
                                        size_t size, void* value, size_t* size_ret) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  switch (name) {
    case CL_QUEUE_CONTEXT: return get_info<cl_context>(q->ctx, size, value, size_ret);
    case CL_QUEUE_DEVICE: return get_info<cl_device_id>(q->dev, size, value, size_ret);
    case CL_QUEUE_REFERENCE_COUNT: return get_info<cl_uint>(q->ref.load(), size, value, size_ret);
    case CL_QUEUE_PROPERTIES:
      return get_info<cl_command_queue_properties>(q->props, size, value, size_ret);
    default: return CL_INVALID_VALUE;
  }
}

extern "C" cl_int clFlush(cl_command_queue q) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  return CL_SUCCESS;  // CUDA submits at launch
}

extern "C" cl_int clFinish(cl_command_queue q) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  cl_int st;
  {
    DeviceGuard g(q->dev->ordinal);
    st = cuda_err(cudaStreamSynchronize(q->stream));
  }
  reap_frees(false);
  return st;
}

// ===================================================================== memory objects
static void* raw_alloc(size_t bytes, int ordinal, cudaStream_t stream, int* kind, bool ipc) {
  DeviceGuard g(ordinal);
  if (g_alloc && !ipc) {
    void* p = g_alloc(bytes, ordinal, stream);
    if (p) {
      *kind = 2;
      return p;
    }
    return nullptr;
  }
  void* p = nullptr;
  if (cudaMalloc(&p, bytes) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  *kind = 1;
  return p;
}

static void raw_free(Store& s) {
  DeviceGuard g(s.ordinal);
  if (s.kind == 1) cudaFree(s.ptr);
  else if (s.kind == 2 && g_free) g_free(s.ptr, s.ordinal, nullptr);
  else if (s.kind == 4) cudaIpcCloseMemHandle(s.ptr);
  s.ptr = nullptr;
  s.kind = 0;
}

// the object's LOCAL store on `ordinal` (never an IPC-imported one)
static Store* find_store(cl_mem m, int ordinal) {
  for (auto& s : m->stores)
    if (s.ordinal == ordinal && s.kind != 4) return &s;
  return nullptr;
}

// ---- deferred, stream-ordered frees (clReleaseMemObject) ----
// The last release of an object records an event on every live queue that
// enqueued work on it and parks its stores here; they are freed once all of
// those events have completed -- checked without blocking on later API calls
// (allocations, releases, clFinish), and with blocking at the last context
// release.  The host never waits in clReleaseMemObject.
struct PendingFree {
  std::vector<Store> stores;
  std::vector<std::pair<int, cudaEvent_t>> events;  // (device, event)
};
static std::mutex g_pend_mu;
static std::vector<PendingFree> g_pending;

static void reap_frees(bool block) {
  std::vector<PendingFree> done;
  {
    std::lock_guard<std::mutex> g(g_pend_mu);
    for (size_t i = 0; i < g_pending.size();) {
      bool ready = true;
      for (auto& e : g_pending[i].events) {
        DeviceGuard dg(e.first);
        const cudaError_t r = block ? cudaEventSynchronize(e.second) : cudaEventQuery(e.second);
        if (r == cudaErrorNotReady) { ready = false; break; }
        cudaGetLastError();  // (an errored event counts as done: the stream is dead)
      }
      if (ready) {
        done.push_back(std::move(g_pending[i]));
        g_pending[i] = std::move(g_pending.back());
        g_pending.pop_back();
      } else {
        ++i;
      }
    }
  }
  for (auto& p : done) {
    for (auto& e : p.events) {
      DeviceGuard dg(e.first);
      cudaEventDestroy(e.second);
    }
    for (auto& st : p.stores) raw_free(st);
  }
}

static cl_mem new_mem(cl_context c, cl_mem_object_type type, cl_mem_flags flags, size_t size) {
  auto* m = new (std::nothrow) _cl_mem();
  if (!m) return nullptr;
  m->ctx = c;
  m->type = type;
  m->flags = flags;
  m->size = size;
  m->alloc_size = (size + 255) / 256 * 256;
  m->stores.reserve(64);  // Store pointers stay valid
  return m;
}

static void register_mem(cl_mem m) {
  m->ctx->ref++;
  std::lock_guard<std::mutex> g(g_mu);
  g_mems.insert(m);
}

static cl_int check_mem_flags(cl_mem_flags flags, void* host_ptr) {
  const cl_mem_flags access = flags & (CL_MEM_READ_WRITE | CL_MEM_WRITE_ONLY | CL_MEM_READ_ONLY);
  if (access && (access & (access - 1))) return CL_INVALID_VALUE;
  const cl_mem_flags known = CL_MEM_READ_WRITE | CL_MEM_WRITE_ONLY | CL_MEM_READ_ONLY |
                             CL_MEM_USE_HOST_PTR | CL_MEM_ALLOC_HOST_PTR | CL_MEM_COPY_HOST_PTR |
                             CL_MEM_HOST_WRITE_ONLY | CL_MEM_HOST_READ_ONLY |
                             CL_MEM_HOST_NO_ACCESS | B2CL_MEM_IPC_EXPORTABLE | B2CL_MEM_TILED_IMAGE;
  if (flags & ~known) return CL_INVALID_VALUE;
  if (flags & CL_MEM_USE_HOST_PTR) return CL_INVALID_VALUE;  // reading A33
  const bool copy = flags & CL_MEM_COPY_HOST_PTR;
  if (copy != (host_ptr != nullptr)) return CL_INVALID_HOST_PTR;
  return CL_SUCCESS;
}

// Allocate the object's storage on `ordinal` if missing (content not valid).
static cl_int ensure_store(cl_mem m, int ordinal, cudaStream_t stream, Store** out) {
  Store* s = find_store(m, ordinal);
  if (!s) {
    reap_frees(false);  // memory of released objects whose users have finished
    int kind = 0;
    void* p = raw_alloc(m->alloc_size, ordinal, stream, &kind,
                        (m->flags & B2CL_MEM_IPC_EXPORTABLE) != 0);
    if (!p) return CL_MEM_OBJECT_ALLOCATION_FAILURE;
    Store st;
    st.ordinal = ordinal;
    st.ptr = static_cast<char*>(p);
    st.kind = kind;
    m->stores.push_back(st);
    s = &m->stores.back();
  }
  *out = s;
  return CL_SUCCESS;
}

extern "C" cl_mem clCreateBuffer(cl_context c, cl_mem_flags flags, size_t size, void* host_ptr,
                                 cl_int* errcode_ret) {
  if (!live(g_contexts, c)) { SET_ERR(CL_INVALID_CONTEXT); return nullptr; }
  cl_int st = check_mem_flags(flags, host_ptr);
  if (st != CL_SUCCESS) { SET_ERR(st); return nullptr; }
  if (flags & B2CL_MEM_TILED_IMAGE) { SET_ERR(CL_INVALID_VALUE); return nullptr; }  // images only
  if (size == 0) { SET_ERR(CL_INVALID_BUFFER_SIZE); return nullptr; }
  cl_mem m = new_mem(c, CL_MEM_OBJECT_BUFFER, flags, size);
  if (!m) { SET_ERR(CL_OUT_OF_HOST_MEMORY); return nullptr; }
  const int ord = c->devs[0]->ordinal;
  Store* s = nullptr;
  st = ensure_store(m, ord, nullptr, &s);
  if (st != CL_SUCCESS) { delete m; SET_ERR(st); return nullptr; }
  if (host_ptr) {
    DeviceGuard g(ord);
    cudaError_t e = cudaMemcpy(s->ptr, host_ptr, size, cudaMemcpyHostToDevice);
    // a pageable-source cudaMemcpy returns once the data is staged, before
    // the DMA lands: wait for it, or a queue's first command (its own
    // stream) could run before the contents exist
    if (e == cudaSuccess) e = cudaStreamSynchronize(nullptr);
    if (e != cudaSuccess) { raw_free(*s); delete m; SET_ERR(cuda_err(e)); return nullptr; }
  }
  m->valid = 1ull << ord;
  register_mem(m);
  SET_ERR(CL_SUCCESS);
  return m;
}

extern "C" cl_mem b2clCreateBufferFromDevicePointer(cl_context c, cl_device_id d, cl_mem_flags flags,
                                                    void* ptr, size_t size, cl_int* errcode_ret) {
  if (!live(g_contexts, c)) { SET_ERR(CL_INVALID_CONTEXT); return nullptr; }
  if (!valid_device(d) || !ctx_has_device(c, d)) { SET_ERR(CL_INVALID_DEVICE); return nullptr; }
  if (!ptr || size == 0 || (flags & (CL_MEM_USE_HOST_PTR | CL_MEM_COPY_HOST_PTR))) {
    SET_ERR(CL_INVALID_VALUE);
    return nullptr;
  }
  cl_mem m = new_mem(c, CL_MEM_OBJECT_BUFFER, flags, size);
  if (!m) { SET_ERR(CL_OUT_OF_HOST_MEMORY); return nullptr; }
  Store s;
  s.ordinal = d->ordinal;
  s.ptr = static_cast<char*>(ptr);
  s.kind = 3;
  m->stores.push_back(s);
  m->valid = 1ull << d->ordinal;
  register_mem(m);
  SET_ERR(CL_SUCCESS);
  return m;
}

// A 1D image buffer ([CL1.2 §5.3.1]): an image view of a buffer's bytes.
static cl_mem image_from_buffer(cl_context c, cl_mem_flags flags, const cl_image_format* fmt,
                                const cl_image_desc* desc, const ImageLayout& L, void* host_ptr,
                                cl_int* errcode_ret) {
  cl_mem b = desc->buffer;
  if (!live(g_mems, b) || b->type != CL_MEM_OBJECT_BUFFER || b->ctx != c) {
    SET_ERR(CL_INVALID_IMAGE_DESCRIPTOR);
    return nullptr;
  }
  // the pixels are the buffer's (no host pointer, no host pitches: reading A34)
  if (host_ptr || (flags & (CL_MEM_COPY_HOST_PTR | CL_MEM_USE_HOST_PTR | CL_MEM_ALLOC_HOST_PTR)) ||
      desc->image_row_pitch || desc->image_slice_pitch) {
    SET_ERR(CL_INVALID_VALUE);
    return nullptr;
  }
  if (L.bytes > b->size) { SET_ERR(CL_INVALID_IMAGE_SIZE); return nullptr; }
  cl_mem m = new_mem(c, CL_MEM_OBJECT_IMAGE1D_BUFFER, flags ? flags : b->flags, L.bytes);
  if (!m) { SET_ERR(CL_OUT_OF_HOST_MEMORY); return nullptr; }
  m->img = L;
  m->fmt = *fmt;
  m->desc = *desc;
  b->ref++;
  m->parent = b;
  register_mem(m);
  SET_ERR(CL_SUCCESS);
  return m;
}

extern "C" cl_mem clCreateImage(cl_context c, cl_mem_flags flags, const cl_image_format* fmt,
                                const cl_image_desc* desc, void* host_ptr, cl_int* errcode_ret) {
  if (!live(g_contexts, c)) { SET_ERR(CL_INVALID_CONTEXT); return nullptr; }
  ImageLayout L;
  cl_int st = image_layout(fmt, desc, &L);
  if (st != CL_SUCCESS) { SET_ERR(st); return nullptr; }
  if (flags & B2CL_MEM_TILED_IMAGE) {  // tiled storage: 2D images only
    if (desc->image_type != CL_MEM_OBJECT_IMAGE2D || !tile_layout(&L)) { SET_ERR(CL_INVALID_VALUE); return nullptr; }
  }
  if (desc->image_type == CL_MEM_OBJECT_IMAGE1D_BUFFER)
    return image_from_buffer(c, flags, fmt, desc, L, host_ptr, errcode_ret);
  st = check_mem_flags(flags & ~(B2CL_MEM_IPC_EXPORTABLE | B2CL_MEM_TILED_IMAGE), host_ptr);
  if (st != CL_SUCCESS) { SET_ERR(st); return nullptr; }
  // host pitches ([CL1.2 §5.3.1]): nonzero only with a host pointer, >= tight,
  // multiple of the element size.  Slice pitch: 3D images and 2D arrays
  // (>= row_pitch * height), 1D arrays (the size of each layer, >= row_pitch),
  // in both cases a multiple of row_pitch; 0 for 1D and 2D images.
  size_t hrp = desc->image_row_pitch, hsp = desc->image_slice_pitch;
  if ((hrp || hsp) && !host_ptr) { SET_ERR(CL_INVALID_IMAGE_DESCRIPTOR); return nullptr; }
  if (hrp == 0) hrp = L.w * L.fmt.es;
  else if (hrp < L.w * L.fmt.es || hrp % L.fmt.es) { SET_ERR(CL_INVALID_IMAGE_DESCRIPTOR); return nullptr; }
  const bool arr1 = L.arrayed && L.dims == 2;
  if (L.dims == 3 || arr1) {
    const size_t min_sp = arr1 ? hrp : hrp * L.h;
    if (hsp == 0) hsp = min_sp;
    else if (hsp < min_sp || hsp % hrp) { SET_ERR(CL_INVALID_IMAGE_DESCRIPTOR); return nullptr; }
    if (arr1) hrp = hsp;  // layer l of a 1D array is host row l, hsp apart
  } else if (hsp != 0) {
    SET_ERR(CL_INVALID_IMAGE_DESCRIPTOR);
    return nullptr;
  }
  cl_mem m = new_mem(c, desc->image_type, flags, L.bytes);
  if (!m) { SET_ERR(CL_OUT_OF_HOST_MEMORY); return nullptr; }
  m->img = L;
  m->fmt = *fmt;
  m->desc = *desc;
  const int ord = c->devs[0]->ordinal;
  Store* s = nullptr;
  st = ensure_store(m, ord, nullptr, &s);
  if (st != CL_SUCCESS) { delete m; SET_ERR(st); return nullptr; }
  if (host_ptr && L.tiled) {  // through a linear staging copy, then tiled on the device
    DeviceGuard g(ord);
    void* stg = nullptr;
    cudaError_t e = cudaMalloc(&stg, L.w * L.fmt.es * L.h);
    if (e == cudaSuccess)
      e = cudaMemcpy2D(stg, L.w * L.fmt.es, host_ptr, hrp, L.w * L.fmt.es, L.h, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) {
      TexCopyParams tp{};
      tp.src.ptr = static_cast<char*>(stg);
      tp.src.rp = L.w * L.fmt.es;
      tp.src.sp = tp.src.rp * L.h;
      tp.dst.ptr = s->ptr;
      tp.dst.rp = L.row_pitch;
      tp.dst.tiled = 1;
      tp.dst.tshift = L.tshift;
      tp.w = (uint32_t)L.w;
      tp.h = (uint32_t)L.h;
      tp.d = 1;
      tp.es = (int)L.fmt.es;
      e = launch_texcopy(tp, nullptr);
      if (e == cudaSuccess) e = cudaStreamSynchronize(nullptr);
    }
    if (stg) cudaFree(stg);
    if (e != cudaSuccess) { raw_free(*s); delete m; SET_ERR(cuda_err(e)); return nullptr; }
  } else if (host_ptr) {  // clCreateImage uploads the contents
    DeviceGuard g(ord);
    for (size_t k = 0; k < L.d; ++k) {
      cudaError_t e = cudaMemcpy2D(s->ptr + k * L.slice_pitch, L.row_pitch,
                                   static_cast<const char*>(host_ptr) + k * hsp, hrp,
                                   L.w * L.fmt.es, L.h, cudaMemcpyHostToDevice);
      if (e != cudaSuccess) { raw_free(*s); delete m; SET_ERR(cuda_err(e)); return nullptr; }
    }
    const cudaError_t e = cudaStreamSynchronize(nullptr);  // (the DMA has landed: see clCreateBuffer)
    if (e != cudaSuccess) { raw_free(*s); delete m; SET_ERR(cuda_err(e)); return nullptr; }
  }
  m->valid = 1ull << ord;
  register_mem(m);
  SET_ERR(CL_SUCCESS);
  return m;
}

extern "C" cl_mem b2clCreateImageShard(cl_context c, cl_mem_flags flags, const cl_image_format* fmt,
                                       const cl_image_desc* global_desc, size_t begin,
                                       size_t count, size_t halo, void* host_ptr,
                                       cl_int* errcode_ret) {
  if (!live(g_contexts, c)) { SET_ERR(CL_INVALID_CONTEXT); return nullptr; }
  if (!global_desc) { SET_ERR(CL_INVALID_IMAGE_DESCRIPTOR); return nullptr; }
  if (flags & B2CL_MEM_TILED_IMAGE) { SET_ERR(CL_INVALID_VALUE); return nullptr; }  // shards are pitched
  ImageLayout G;
  cl_int st = image_layout(fmt, global_desc, &G);
  if (st != CL_SUCCESS) { SET_ERR(st); return nullptr; }
  if (G.dims < 2 || G.arrayed) { SET_ERR(CL_INVALID_IMAGE_DESCRIPTOR); return nullptr; }
  const size_t extent = G.dims == 3 ? G.d : G.h;
  // the band may wrap around the global extent (begin + count > extent)
  if (count == 0 || begin >= extent || count + 2 * halo > extent ||
      global_desc->image_row_pitch || global_desc->image_slice_pitch) {
    SET_ERR(CL_INVALID_VALUE);
    return nullptr;
  }
  // the stored rows as a plain image of count + 2*halo rows (or slices)
  cl_image_desc sd = *global_desc;
  if (G.dims == 3) sd.image_depth = count + 2 * halo;
  else sd.image_height = count + 2 * halo;
  cl_mem m = clCreateImage(c, flags, fmt, &sd, host_ptr, errcode_ret);
  if (!m) return nullptr;
  m->shard = true;
  m->shard_extent = extent;
  m->shard_ob = (long long)begin - (long long)halo;
  return m;
}

extern "C" cl_int clGetSupportedImageFormats(cl_context c, cl_mem_flags flags,
                                             cl_mem_object_type type, cl_uint num_entries,
                                             cl_image_format* formats, cl_uint* num_formats) {
  (void)flags;
  if (!live(g_contexts, c)) return CL_INVALID_CONTEXT;
  if (type < CL_MEM_OBJECT_IMAGE2D || type > CL_MEM_OBJECT_IMAGE1D_BUFFER) return CL_INVALID_VALUE;
  if (num_entries == 0 && formats) return CL_INVALID_VALUE;
  std::vector<cl_image_format> all;
  for (cl_channel_order o = CL_R; o <= CL_RGBx; ++o)
    for (cl_channel_type t = CL_SNORM_INT8; t <= CL_FLOAT; ++t) {
      cl_image_format f{o, t};
      FormatInfo fi;
      if (format_info(&f, &fi) == CL_SUCCESS) all.push_back(f);
    }
  if (formats)
    for (cl_uint i = 0; i < std::min<cl_uint>(num_entries, (cl_uint)all.size()); ++i) formats[i] = all[i];
  if (num_formats) *num_formats = (cl_uint)all.size();
  return CL_SUCCESS;
}

static bool is_image(cl_mem m) {
  return m->type >= CL_MEM_OBJECT_IMAGE2D && m->type <= CL_MEM_OBJECT_IMAGE1D_BUFFER;
}

extern "C" cl_int clRetainMemObject(cl_mem m) {
  return retain_ref(g_mems, m) ? CL_SUCCESS : CL_INVALID_MEM_OBJECT;
}

extern "C" cl_int clReleaseMemObject(cl_mem m) {
  const int r = release_ref(g_mems, m);
  if (r < 0) return CL_INVALID_MEM_OBJECT;
  if (r == 1) {
    // stream-ordered, deferred free (ownership): an event after
    // the object's last command on every queue that used it; the stores are
    // freed once they complete (reap_frees) -- no host wait here
    std::vector<cl_command_queue> users;
    {
      std::lock_guard<std::mutex> gm(m->mu);
      users.assign(m->users.begin(), m->users.end());
    }
    PendingFree pf;
    {
      std::lock_guard<std::mutex> g(g_mu);  // queues stay alive while recording
      for (cl_command_queue q : users) {
        if (!g_queues.count(q)) continue;  // released queues were drained then
        DeviceGuard dg(q->dev->ordinal);
        cudaEvent_t ev = nullptr;
        if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) == cudaSuccess &&
            cudaEventRecord(ev, q->stream) == cudaSuccess) {
          pf.events.emplace_back(q->dev->ordinal, ev);
        } else {  // no event: fall back to draining that queue
          if (ev) cudaEventDestroy(ev);
          cudaGetLastError();
          cudaStreamSynchronize(q->stream);
        }
      }
    }
    pf.stores = std::move(m->stores);
    if (!pf.stores.empty()) {
      std::lock_guard<std::mutex> g(g_pend_mu);
      g_pending.push_back(std::move(pf));
    }
    cl_context c = m->ctx;
    cl_mem parent = m->parent;
    delete m;
    if (parent) clReleaseMemObject(parent);
    reap_frees(false);
    clReleaseContext(c);
  }
  return CL_SUCCESS;
}

extern "C" cl_int clGetMemObjectInfo(cl_mem m, cl_mem_info name, size_t size, void* value,
                                     size_t* size_ret) {
  if (!live(g_mems, m)) return CL_INVALID_MEM_OBJECT;
  switch (name) {
    case CL_MEM_TYPE: return get_info<cl_mem_object_type>(m->type, size, value, size_ret);
    case CL_MEM_FLAGS: return get_info<cl_mem_flags>(m->flags, size, value, size_ret);
    case CL_MEM_SIZE: return get_info<size_t>(m->size, size, value, size_ret);
    case CL_MEM_HOST_PTR: return get_info<void*>(nullptr, size, value, size_ret);
    case CL_MEM_MAP_COUNT: return get_info<cl_uint>(0, size, value, size_ret);
    case CL_MEM_REFERENCE_COUNT: return get_info<cl_uint>(m->ref.load(), size, value, size_ret);
    case CL_MEM_CONTEXT: return get_info<cl_context>(m->ctx, size, value, size_ret);
    case CL_MEM_ASSOCIATED_MEMOBJECT: return get_info<cl_mem>(m->parent, size, value, size_ret);
    case CL_MEM_OFFSET: return get_info<size_t>(0, size, value, size_ret);
    default: return CL_INVALID_VALUE;
  }
}

extern "C" cl_int clGetImageInfo(cl_mem m, cl_image_info name, size_t size, void* value,
                                 size_t* size_ret) {
  if (!live(g_mems, m) || !is_image(m)) return CL_INVALID_MEM_OBJECT;
  const ImageLayout& L = m->img;
  switch (name) {
    case CL_IMAGE_FORMAT: return get_info<cl_image_format>(m->fmt, size, value, size_ret);
    case CL_IMAGE_ELEMENT_SIZE: return get_info<size_t>(L.fmt.es, size, value, size_ret);
    case CL_IMAGE_ROW_PITCH:  // (tiled storage: the pitch of its linear view, reading A46)
      return get_info<size_t>(L.tiled ? L.w * L.fmt.es : L.row_pitch, size, value, size_ret);
    case CL_IMAGE_SLICE_PITCH: {
      // 3D: bytes per slice; arrays: bytes per layer; 1D, 1D buffer and 2D: 0
      const size_t sp = (L.dims == 3) ? L.slice_pitch : (L.arrayed ? L.row_pitch : 0);
      return get_info<size_t>(sp, size, value, size_ret);
    }
    case CL_IMAGE_WIDTH: return get_info<size_t>(L.w, size, value, size_ret);
    case CL_IMAGE_HEIGHT:
      return get_info<size_t>(L.dims - L.arrayed > 1 ? L.h : 0, size, value, size_ret);
    case CL_IMAGE_DEPTH:
      return get_info<size_t>(L.dims == 3 && !L.arrayed ? L.d : 0, size, value, size_ret);
    case CL_IMAGE_ARRAY_SIZE:
      return get_info<size_t>(!L.arrayed ? 0 : (L.dims == 2 ? L.h : L.d), size, value, size_ret);
    case CL_IMAGE_BUFFER: return get_info<cl_mem>(m->parent, size, value, size_ret);
    case CL_IMAGE_NUM_MIP_LEVELS:
    case CL_IMAGE_NUM_SAMPLES: return get_info<cl_uint>(0, size, value, size_ret);
    default: return CL_INVALID_VALUE;
  }
}

extern "C" cl_int b2clSetAllocator(b2cl_alloc_fn a, b2cl_free_fn f) {
  if ((a == nullptr) != (f == nullptr)) return CL_INVALID_VALUE;
  g_alloc = a;
  g_free = f;
  return CL_SUCCESS;
}

// ===================================================================== sampler
extern "C" cl_sampler clCreateSampler(cl_context c, cl_bool norm, cl_addressing_mode am,
                                      cl_filter_mode fm, cl_int* errcode_ret) {
  if (!live(g_contexts, c)) { SET_ERR(CL_INVALID_CONTEXT); return nullptr; }
  cl_int st = validate_sampler(norm, am, fm);
  if (st != CL_SUCCESS) { SET_ERR(st); return nullptr; }
  auto* s = new (std::nothrow) _cl_sampler();
  if (!s) { SET_ERR(CL_OUT_OF_HOST_MEMORY); return nullptr; }
  s->ctx = c;
  s->norm = norm;
  s->addr = am;
  s->filt = fm;
  c->ref++;
  {
    std::lock_guard<std::mutex> g(g_mu);
    g_samplers.insert(s);
  }
  SET_ERR(CL_SUCCESS);
  return s;
}

extern "C" cl_int clRetainSampler(cl_sampler s) {
  return retain_ref(g_samplers, s) ? CL_SUCCESS : CL_INVALID_SAMPLER;
}

extern "C" cl_int clReleaseSampler(cl_sampler s) {
  const int r = release_ref(g_samplers, s);
  if (r < 0) return CL_INVALID_SAMPLER;
  if (r == 1) {
    cl_context c = s->ctx;
    delete s;
    clReleaseContext(c);
  }
  return CL_SUCCESS;
}

extern "C" cl_int clGetSamplerInfo(cl_sampler s, cl_sampler_info name, size_t size, void* value,
                                   size_t* size_ret) {
  if (!live(g_samplers, s)) return CL_INVALID_SAMPLER;
  switch (name) {
    case CL_SAMPLER_REFERENCE_COUNT: return get_info<cl_uint>(s->ref.load(), size, value, size_ret);
    case CL_SAMPLER_CONTEXT: return get_info<cl_context>(s->ctx, size, value, size_ret);
    case CL_SAMPLER_NORMALIZED_COORDS: return get_info<cl_bool>(s->norm, size, value, size_ret);
    case CL_SAMPLER_ADDRESSING_MODE: return get_info<cl_addressing_mode>(s->addr, size, value, size_ret);
    case CL_SAMPLER_FILTER_MODE: return get_info<cl_filter_mode>(s->filt, size, value, size_ret);
    default: return CL_INVALID_VALUE;
  }
}

// ===================================================================== events
extern "C" cl_int clWaitForEvents(cl_uint n, const cl_event* list) {
  if (n == 0 || !list) return CL_INVALID_VALUE;
  for (cl_uint i = 0; i < n; ++i)
    if (!live(g_events, list[i])) return CL_INVALID_EVENT;
  for (cl_uint i = 0; i < n; ++i) {
    cudaError_t e = cudaEventSynchronize(list[i]->end);
    if (e != cudaSuccess) return cuda_err(e);
  }
  return CL_SUCCESS;
}

extern "C" cl_int clRetainEvent(cl_event e) {
  return retain_ref(g_events, e) ? CL_SUCCESS : CL_INVALID_EVENT;
}

extern "C" cl_int clReleaseEvent(cl_event e) {
  const int r = release_ref(g_events, e);
  if (r < 0) return CL_INVALID_EVENT;
  if (r == 1) {
    DeviceGuard g(e->ordinal);
    if (e->start) cudaEventDestroy(e->start);
    if (e->end) cudaEventDestroy(e->end);
    cl_context c = e->ctx;
    delete e;
    clReleaseContext(c);
  }
  return CL_SUCCESS;
}

extern "C" cl_int clGetEventInfo(cl_event e, cl_event_info name, size_t size, void* value,
                                 size_t* size_ret) {
  if (!live(g_events, e)) return CL_INVALID_EVENT;
  switch (name) {
    case CL_EVENT_COMMAND_QUEUE: return get_info<cl_command_queue>(e->queue, size, value, size_ret);
    case CL_EVENT_CONTEXT: return get_info<cl_context>(e->ctx, size, value, size_ret);
    case CL_EVENT_COMMAND_TYPE: return get_info<cl_command_type>(e->type, size, value, size_ret);
    case CL_EVENT_REFERENCE_COUNT: return get_info<cl_uint>(e->ref.load(), size, value, size_ret);
    case CL_EVENT_COMMAND_EXECUTION_STATUS: {
      cudaError_t q = cudaEventQuery(e->end);
      cl_int status = q == cudaSuccess ? CL_COMPLETE : CL_SUBMITTED;
      if (q != cudaSuccess && q != cudaErrorNotReady) status = CL_OUT_OF_RESOURCES;
      cudaGetLastError();
      return get_info<cl_int>(status, size, value, size_ret);
    }
    default: return CL_INVALID_VALUE;
  }
}

extern "C" cl_int clGetEventProfilingInfo(cl_event e, cl_profiling_info name, size_t size,
                                          void* value, size_t* size_ret) {
  if (!live(g_events, e)) return CL_INVALID_EVENT;
  if (!e->start) return CL_PROFILING_INFO_NOT_AVAILABLE;
  if (cudaEventQuery(e->end) != cudaSuccess) {
    cudaGetLastError();
    return CL_PROFILING_INFO_NOT_AVAILABLE;
  }
  float ms = 0.f;
  cudaEvent_t which = name == CL_PROFILING_COMMAND_END ? e->end : e->start;
  if (name < CL_PROFILING_COMMAND_QUEUED || name > CL_PROFILING_COMMAND_END) return CL_INVALID_VALUE;
  DeviceGuard g(e->ordinal);
  if (cudaEventElapsedTime(&ms, g_epoch[e->ordinal], which) != cudaSuccess) {
    cudaGetLastError();
    return CL_PROFILING_INFO_NOT_AVAILABLE;
  }
  return get_info<cl_ulong>((cl_ulong)((double)ms * 1e6), size, value, size_ret);
}

// ===================================================================== enqueue plumbing
struct Enq {
  cl_command_queue q = nullptr;
  cl_event* evout = nullptr;
  cl_command_type type = 0;
  cudaEvent_t start = nullptr;
  uint64_t launches0 = 0;  // library launch count at enq_begin (tracing)
};

static cl_int check_wait_list(cl_command_queue q, cl_uint n, const cl_event* list) {
  if ((n == 0) != (list == nullptr)) return CL_INVALID_EVENT_WAIT_LIST;
  for (cl_uint i = 0; i < n; ++i)
    if (!live(g_events, list[i]) || list[i]->ctx != q->ctx) return CL_INVALID_EVENT_WAIT_LIST;
  return CL_SUCCESS;
}

// after validation: make the stream wait for the wait list; start event
static cl_int enq_begin(Enq& E, cl_uint n, const cl_event* list) {
  E.launches0 = launch_count();
  for (cl_uint i = 0; i < n; ++i) cudaStreamWaitEvent(E.q->stream, list[i]->end, 0);
  if (E.evout && (E.q->props & CL_QUEUE_PROFILING_ENABLE)) {
    if (cudaEventCreate(&E.start) != cudaSuccess) return CL_OUT_OF_RESOURCES;
    cudaEventRecord(E.start, E.q->stream);
  }
  return CL_SUCCESS;
}

// ---- tracing: B2CL_LOG=1 prints one line per enqueued command
// to stderr (command, queue, device, the kernel the library picked, status);
// B2CL_NVTX=1 drops an NVTX mark with the same text (nsys / ncu --nvtx).
static const char* command_name(cl_command_type t) {
  switch (t) {
    case CL_COMMAND_NDRANGE_KERNEL: return "NDRANGE_KERNEL";
    case CL_COMMAND_READ_BUFFER: return "READ_BUFFER";
    case CL_COMMAND_WRITE_BUFFER: return "WRITE_BUFFER";
    case CL_COMMAND_COPY_BUFFER: return "COPY_BUFFER";
    case CL_COMMAND_READ_IMAGE: return "READ_IMAGE";
    case CL_COMMAND_WRITE_IMAGE: return "WRITE_IMAGE";
    case CL_COMMAND_COPY_IMAGE: return "COPY_IMAGE";
    case CL_COMMAND_COPY_IMAGE_TO_BUFFER: return "COPY_IMAGE_TO_BUFFER";
    case CL_COMMAND_COPY_BUFFER_TO_IMAGE: return "COPY_BUFFER_TO_IMAGE";
    case CL_COMMAND_MARKER: return "MARKER";
    case CL_COMMAND_READ_BUFFER_RECT: return "READ_BUFFER_RECT";
    case CL_COMMAND_WRITE_BUFFER_RECT: return "WRITE_BUFFER_RECT";
    case CL_COMMAND_COPY_BUFFER_RECT: return "COPY_BUFFER_RECT";
    case CL_COMMAND_BARRIER: return "BARRIER";
    case CL_COMMAND_MIGRATE_MEM_OBJECTS: return "MIGRATE_MEM_OBJECTS";
    case CL_COMMAND_FILL_BUFFER: return "FILL_BUFFER";
    case CL_COMMAND_FILL_IMAGE: return "FILL_IMAGE";
    default: return "COMMAND";
  }
}

static void trace_command(const Enq& E, cl_int status) {
  static const int log = getenv("B2CL_LOG") ? atoi(getenv("B2CL_LOG")) : 0;
  static const int nvtx = getenv("B2CL_NVTX") ? atoi(getenv("B2CL_NVTX")) : 0;
  if (!log && !nvtx) return;
  char buf[160];
  snprintf(buf, sizeof(buf), "b2cl %s queue=%p dev=%d kernel=%s status=%d", command_name(E.type),
           static_cast<void*>(E.q), E.q->dev->ordinal, launch_count() > E.launches0 ? last_kernel() : "-",
           status);
  if (log) fprintf(stderr, "[%s]\n", buf);
  if (nvtx) nvtxMarkA(buf);
}

static cl_int enq_end(Enq& E, cudaError_t err) {
  trace_command(E, err == cudaSuccess ? CL_SUCCESS : cuda_err(err));
  if (err != cudaSuccess) {
    if (E.start) cudaEventDestroy(E.start);
    return cuda_err(err);
  }
  if (E.evout) {
    auto* ev = new (std::nothrow) _cl_event();
    if (!ev) return CL_OUT_OF_HOST_MEMORY;
    ev->ctx = E.q->ctx;
    ev->queue = E.q;
    ev->type = E.type;
    ev->ordinal = E.q->dev->ordinal;
    ev->start = E.start;
    const unsigned flags = E.start ? cudaEventDefault : cudaEventDisableTiming;
    if (cudaEventCreateWithFlags(&ev->end, flags) != cudaSuccess) {
      delete ev;
      return CL_OUT_OF_RESOURCES;
    }
    cudaEventRecord(ev->end, E.q->stream);
    E.q->ctx->ref++;
    {
      std::lock_guard<std::mutex> g(g_mu);
      g_events.insert(ev);
    }
    *E.evout = ev;
  }
  return CL_SUCCESS;
}

// Can queue q's device address store st directly?  Its own memory; a peer
// GPU's with peer access enabled in the context (NVLink); an IPC mapping
// opened on this device.
static bool reachable(cl_command_queue q, const Store& st) {
  const int ord = q->dev->ordinal;
  if (st.kind == 4 || st.ordinal == ord) return st.ordinal == ord;
  return st.ordinal >= 0 && st.ordinal < 64 && q->ctx->peer[ord][st.ordinal];
}

// Copy the object's whole valid content into the store `dst` of q's device
// on q's stream (the caller has issued the wait list first: enq_begin).
static cudaError_t pull_whole(cl_mem m, cl_command_queue q, Store* dst) {
  Store* src = nullptr;
  for (auto& o : m->stores)
    if (((m->valid >> bit_of(o)) & 1ull) && &o != dst) { src = &o; break; }
  if (!src) return cudaSuccess;
  if (reachable(q, *src)) {  // SM copy kernel reading the peer / IPC pointer (NVLink)
    RectParams p{};
    p.src = src->ptr;
    p.dst = dst->ptr;
    p.R0 = m->alloc_size;
    p.R1 = p.R2 = 1;
    p.srp = p.drp = m->alloc_size;
    p.ssp = p.dsp = m->alloc_size;
    return launch_rect(p, RECT_COPY, q->stream);
  }
  return cudaMemcpyPeerAsync(dst->ptr, dst->ordinal, src->ptr, src->ordinal, m->alloc_size, q->stream);
}

// Make the object's content valid on the queue's device and return its
// pointer there.  If another device (or another process, through an IPC
// mapping) holds the only valid copy, pull it whole over NVLink on the
// queue's stream.  Callers issue the wait list (enq_begin) BEFORE this, so the
// pull is ordered after the producer of the content (OpenCL cross-queue rule).
static cl_int resident(cl_mem m, cl_command_queue q, bool need_content, char** out) {
  size_t off = 0;
  if (m->parent) {  // a 1D image buffer or a view lives in its parent
    off = m->parent_off;
    m = m->parent;
  }
  std::lock_guard<std::mutex> g(m->mu);
  const int ord = q->dev->ordinal;
  Store* s = nullptr;
  cl_int st = ensure_store(m, ord, q->stream, &s);
  if (st != CL_SUCCESS) return st;
  const uint64_t bit = 1ull << ord;
  if (need_content && !(m->valid & bit) && m->valid) {
    const cudaError_t e = pull_whole(m, q, s);
    if (e != cudaSuccess) return cuda_err(e);
    m->valid |= bit;
  }
  m->users.insert(q);
  *out = s->ptr + off;
  return CL_SUCCESS;
}

// Region copies and fills touch part of an object, so they address a valid
// copy IN PLACE when q's device can reach it -- a source region is read from
// the peer (NVLink) or IPC pointer, a destination region written there --
// with no whole-object migration and no full-size allocation (a halo row
// exchanged between two shards moves the row, not the shard).  Only when no
// reachable copy is valid does the object migrate to q's device.
// *store is the store written (for `written_store`).
static cl_int in_place(cl_mem m, cl_command_queue q, bool for_write, char** out, Store** store) {
  size_t off = 0;
  if (m->parent) {
    off = m->parent_off;
    m = m->parent;
  }
  std::lock_guard<std::mutex> g(m->mu);
  const int ord = q->dev->ordinal;
  m->users.insert(q);
  Store* local = find_store(m, ord);
  Store* pick = nullptr;
  if (local && (m->valid & (1ull << ord))) {
    pick = local;
  } else if (m->valid) {
    for (auto& o : m->stores)
      if (((m->valid >> bit_of(o)) & 1ull) && reachable(q, o)) { pick = &o; break; }
  }
  if (!pick) {  // nothing valid (fresh object) or nothing reachable: a local copy
    cl_int st = ensure_store(m, ord, q->stream, &local);
    if (st != CL_SUCCESS) return st;
    if (m->valid) {
      const cudaError_t e = pull_whole(m, q, local);
      if (e != cudaSuccess) return cuda_err(e);
    }
    if (m->valid || !for_write) m->valid |= 1ull << ord;
    pick = local;
  }
  *out = pick->ptr + off;
  if (store) *store = pick;
  return CL_SUCCESS;
}

static void written(cl_mem m, cl_command_queue q) {
  if (m->parent) m = m->parent;
  std::lock_guard<std::mutex> g(m->mu);
  m->valid = 1ull << q->dev->ordinal;
}

// after a write through in_place: the written store is the only valid copy
static void written_store(cl_mem m, const Store* st) {
  if (m->parent) m = m->parent;
  std::lock_guard<std::mutex> g(m->mu);
  m->valid = 1ull << bit_of(*st);
}

// an error after enq_begin: drop the profiling start event (the wait-list
// waits it issued only order the stream; nothing else was enqueued)
static cl_int enq_fail(Enq& E, cl_int st) {
  if (E.start) cudaEventDestroy(E.start);
  E.start = nullptr;
  return st;
}

#define CHECK_E(E, x)                        \
  do {                                       \
    cl_int _s = (x);                         \
    if (_s != CL_SUCCESS) return enq_fail(E, _s); \
  } while (0)

static cl_int check_queue_mem(cl_command_queue q, cl_mem m) {
  if (!live(g_mems, m) || m->ctx != q->ctx) return CL_INVALID_MEM_OBJECT;
  return CL_SUCCESS;
}

#define CHECK(x)                        \
  do {                                  \
    cl_int _s = (x);                    \
    if (_s != CL_SUCCESS) return _s;    \
  } while (0)

// ---- CUDA texture front end (b2cl_ext.h, reading A40) ----
// An image view: layout L over the storage of `parent` (a buffer or an
// image) from byte `off` on; retains the parent, owns no storage.
static cl_mem image_view(cl_context c, cl_mem parent, size_t off, cl_mem_object_type type,
                         const cl_image_format& fmt, const ImageLayout& L) {
  if (parent->parent) {  // views of views share the root storage
    off += parent->parent_off;
    parent = parent->parent;
  }
  cl_mem m = new_mem(c, type, parent->flags & (CL_MEM_READ_WRITE | CL_MEM_WRITE_ONLY | CL_MEM_READ_ONLY),
                     L.bytes);
  if (!m) return nullptr;
  m->img = L;
  m->fmt = fmt;
  m->desc.image_type = type;
  m->desc.image_width = L.w;
  m->desc.image_height = L.arrayed && L.dims == 2 ? 0 : L.h;
  m->desc.image_depth = L.dims == 3 && !L.arrayed ? L.d : 0;
  m->desc.image_array_size = L.arrayed ? (L.dims == 2 ? L.h : L.d) : 0;
  parent->ref++;
  m->parent = parent;
  m->parent_off = off;
  register_mem(m);
  return m;
}

extern "C" cl_int b2clCreateTextureObject(cl_context c, const b2cl_resource_desc* rd,
                                          const b2cl_texture_desc* td, b2cl_texture* tex) {
  if (!live(g_contexts, c)) return CL_INVALID_CONTEXT;
  if (!rd || !td || !tex) return CL_INVALID_VALUE;
  if (!live(g_mems, rd->mem) || rd->mem->ctx != c) return CL_INVALID_MEM_OBJECT;
  cl_mem src = rd->mem;
  cl_image_format stored{};
  ImageLayout L{};
  cl_mem_object_type vtype = 0;
  cl_uint sdims = 1;  // sampled axes
  if (rd->res_type == B2CL_RESOURCE_ARRAY) {
    if (!is_image(src) || src->shard || src->type == CL_MEM_OBJECT_IMAGE1D_BUFFER || src->img.tiled)
      return CL_INVALID_MEM_OBJECT;
    stored = src->fmt;
    L = src->img;
    vtype = src->type;
    sdims = (cl_uint)(L.dims - L.arrayed);
  } else if (rd->res_type == B2CL_RESOURCE_LINEAR || rd->res_type == B2CL_RESOURCE_PITCH2D) {
    if (src->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_MEM_OBJECT;
    CHECK(channel_format(&rd->desc, &stored));
    cl_image_desc d{};
    const bool lin = rd->res_type == B2CL_RESOURCE_LINEAR;
    FormatInfo fi;
    CHECK(format_info(&stored, &fi));
    d.image_type = lin ? CL_MEM_OBJECT_IMAGE1D_BUFFER : CL_MEM_OBJECT_IMAGE2D;
    d.image_width = lin ? rd->size_in_bytes / fi.es : rd->width;
    d.image_height = lin ? 0 : rd->height;
    d.buffer = lin ? src : nullptr;
    if (lin && rd->size_in_bytes % fi.es) return CL_INVALID_VALUE;
    CHECK(image_layout(&stored, &d, &L));
    if (!lin) {  // the caller's pitch, not the internal one
      if (rd->pitch_in_bytes < L.w * fi.es || rd->pitch_in_bytes % fi.es) return CL_INVALID_VALUE;
      L.row_pitch = rd->pitch_in_bytes;
      L.slice_pitch = L.row_pitch * L.h;
      L.bytes = L.row_pitch * (L.h - 1) + L.w * fi.es;
    }
    // texels naturally aligned (buffers start 256-byte aligned) and inside the buffer
    if (rd->offset % fi.es || rd->offset > src->size || L.bytes > src->size - rd->offset)
      return CL_INVALID_VALUE;
    vtype = d.image_type;
    sdims = 1 + (lin ? 0 : 1);
  } else {
    return CL_INVALID_VALUE;
  }
  cl_image_format view{};
  cl_bool nc;
  cl_addressing_mode am;
  cl_filter_mode fm;
  b2cl_rtype rt;
  CHECK(texture_mapping(td, sdims, &stored, &view, &nc, &am, &fm, &rt));
  FormatInfo vfi;
  CHECK(format_info(&view, &vfi));
  L.fmt = vfi;  // same bits per texel: only the read conversion changes
  cl_mem img = nullptr;
  if (rd->res_type == B2CL_RESOURCE_ARRAY && view.image_channel_data_type == stored.image_channel_data_type) {
    img = src;  // the image itself
    src->ref++;
  } else {
    img = image_view(c, src, rd->res_type == B2CL_RESOURCE_ARRAY ? 0 : rd->offset, vtype, view, L);
    if (!img) return CL_OUT_OF_HOST_MEMORY;
  }
  cl_sampler smp = nullptr;
  if (rd->res_type != B2CL_RESOURCE_LINEAR) {  // tex1Dfetch takes no sampler
    cl_int st = CL_SUCCESS;
    smp = clCreateSampler(c, nc, am, fm, &st);
    if (!smp) {
      clReleaseMemObject(img);
      return st;
    }
  }
  tex->image = img;
  tex->sampler = smp;
  tex->rtype = rt;
  return CL_SUCCESS;
}

extern "C" cl_int b2clDestroyTextureObject(b2cl_texture* tex) {
  if (!tex) return CL_INVALID_VALUE;
  if (tex->image && !live(g_mems, tex->image)) return CL_INVALID_MEM_OBJECT;
  if (tex->sampler && !live(g_samplers, tex->sampler)) return CL_INVALID_SAMPLER;
  if (tex->image) clReleaseMemObject(tex->image);
  if (tex->sampler) clReleaseSampler(tex->sampler);
  tex->image = nullptr;
  tex->sampler = nullptr;
  return CL_SUCCESS;
}


// Device view of an image.  For the read built-ins (sampling) a shard
// presents its global extent on the outer axis with the stored window (ob,
// os); every other operation addresses the stored rows as a plain image.
static dev::Image dev_image(cl_mem m, char* ptr, bool sampling = false) {
  dev::Image im{};
  const ImageLayout& L = m->img;
  im.ptr = ptr;
  im.w = (int)L.w;
  im.h = (int)L.h;
  im.d = (int)L.d;
  im.type = L.fmt.type;
  im.order = L.fmt.order;
  im.es = (int)L.fmt.es;
  im.nch = L.fmt.nch;
  im.rp = L.row_pitch;
  im.sp = L.slice_pitch;
  im.ob = 0;
  im.os = L.dims == 3 ? im.d : im.h;
  im.tiled = L.tiled;
  im.tshift = L.tshift;
  if (sampling && m->shard) {
    im.ob = (int)m->shard_ob;
    if (L.dims == 3) im.d = (int)m->shard_extent;
    else im.h = (int)m->shard_extent;
  }
  return im;
}

// ===================================================================== tiled images
// A pixel box of an image as one side of k_texcopy (the box origin `o`, texels).
static TexSide image_side(cl_mem m, char* base, const size_t* o) {
  const ImageLayout& L = m->img;
  TexSide t{};
  t.rp = L.row_pitch;
  t.sp = L.slice_pitch;
  if (L.tiled) {
    t.ptr = base;
    t.tiled = 1;
    t.tshift = L.tshift;
    t.ox = (int)o[0];
    t.oy = (int)o[1];
  } else {
    t.ptr = base + o[2] * L.slice_pitch + o[1] * L.row_pitch + o[0] * L.fmt.es;
  }
  return t;
}

static TexSide linear_side(char* p, size_t rp, size_t sp) {
  TexSide t{};
  t.ptr = p;
  t.rp = rp;
  t.sp = sp;
  return t;
}

// One k_texcopy between memory objects (at least one a tiled image): the
// wait list, then the objects addressed in place (A44), then the kernel.
// `build` fills the parameters from the resolved base pointers.
static cl_int tex_enqueue(cl_command_queue q, cl_mem src, cl_mem dst,
                          const std::function<void(char*, char*, TexCopyParams&)>& build, cl_uint nw,
                          const cl_event* wl, cl_event* ev, cl_command_type type) {
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = type;
  DeviceGuard g(q->dev->ordinal);
  char *s = nullptr, *d = nullptr;
  Store* ds = nullptr;
  CHECK(enq_begin(E, nw, wl));
  if (src) CHECK_E(E, in_place(src, q, false, &s, nullptr));
  CHECK_E(E, in_place(dst, q, true, &d, &ds));
  TexCopyParams p{};
  build(s, d, p);
  const cl_int st = enq_end(E, launch_texcopy(p, q->stream));
  if (st == CL_SUCCESS) written_store(dst, ds);
  return st;
}

// Read/WriteImage of a tiled image: the host rows go through a linear
// staging buffer on the queue's stream (stream-ordered allocation), tiled or
// untiled on the device by k_texcopy.
static cl_int tiled_image_host(cl_command_queue q, cl_mem img, cl_bool blocking, const size_t* origin,
                               const size_t* region, size_t hrp, size_t hsp, char* ptr, bool write, cl_uint nw,
                               const cl_event* wl, cl_event* ev) {
  CHECK(check_wait_list(q, nw, wl));
  const ImageLayout& L = img->img;
  const size_t es = L.fmt.es, row = region[0] * es, bytes = row * region[1] * region[2];
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = write ? CL_COMMAND_WRITE_IMAGE : CL_COMMAND_READ_IMAGE;
  DeviceGuard g(q->dev->ordinal);
  CHECK(enq_begin(E, nw, wl));
  char* d = nullptr;
  Store* ds = nullptr;
  CHECK_E(E, write ? in_place(img, q, true, &d, &ds) : resident(img, q, true, &d));
  void* stg = nullptr;
  cudaError_t e = cudaMallocAsync(&stg, bytes, q->stream);
  if (e != cudaSuccess) return enq_fail(E, cuda_err(e));
  TexCopyParams p{};
  p.w = (uint32_t)region[0];
  p.h = (uint32_t)region[1];
  p.d = (uint32_t)region[2];
  p.es = (int)es;
  const TexSide lin = linear_side(static_cast<char*>(stg), row, row * region[1]);
  const TexSide im = image_side(img, d, origin);
  if (write) {
    for (size_t k = 0; k < region[2] && e == cudaSuccess; ++k)
      e = cudaMemcpy2DAsync(static_cast<char*>(stg) + k * row * region[1], row, ptr + k * hsp, hrp, row, region[1],
                            cudaMemcpyHostToDevice, q->stream);
    p.src = lin;
    p.dst = im;
    if (e == cudaSuccess) e = launch_texcopy(p, q->stream);
  } else {
    p.src = im;
    p.dst = lin;
    e = launch_texcopy(p, q->stream);
    for (size_t k = 0; k < region[2] && e == cudaSuccess; ++k)
      e = cudaMemcpy2DAsync(ptr + k * hsp, hrp, static_cast<char*>(stg) + k * row * region[1], row, row, region[1],
                            cudaMemcpyDeviceToHost, q->stream);
  }
  cudaFreeAsync(stg, q->stream);
  cl_int st = enq_end(E, e);
  if (st != CL_SUCCESS) return st;
  if (write) written_store(img, ds);
  if (blocking) return cuda_err(cudaStreamSynchronize(q->stream));
  return CL_SUCCESS;
}

// ===================================================================== host <-> device transfers
static cl_int host_rect_copy(Enq& E, char* dev, size_t drp, size_t dsp, char* host, size_t hrp,
                             size_t hsp, const size_t* region, bool to_device, cl_bool blocking) {
  DeviceGuard g(E.q->dev->ordinal);
  cudaError_t e = cudaSuccess;
  for (size_t k = 0; k < region[2] && e == cudaSuccess; ++k) {
    if (to_device)
      e = cudaMemcpy2DAsync(dev + k * dsp, drp, host + k * hsp, hrp, region[0], region[1],
                            cudaMemcpyHostToDevice, E.q->stream);
    else
      e = cudaMemcpy2DAsync(host + k * hsp, hrp, dev + k * dsp, drp, region[0], region[1],
                            cudaMemcpyDeviceToHost, E.q->stream);
  }
  cl_int st = enq_end(E, e);
  if (st != CL_SUCCESS) return st;
  if (blocking) return cuda_err(cudaStreamSynchronize(E.q->stream));
  return CL_SUCCESS;
}

static cl_int buffer_host_rect(cl_command_queue q, cl_mem buf, cl_bool blocking, const size_t* bo,
                               const size_t* ho, const size_t* region, size_t brp, size_t bsp,
                               size_t hrp, size_t hsp, char* ptr, bool write, cl_uint nw,
                               const cl_event* wl, cl_event* ev, cl_command_type type) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, buf));
  if (buf->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_MEM_OBJECT;
  if (!ptr) return CL_INVALID_VALUE;
  CHECK(validate_host_rect(buf->size, bo, ho, region, brp, bsp, hrp, hsp));
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = type;
  DeviceGuard g(q->dev->ordinal);
  char* d = nullptr;
  CHECK(enq_begin(E, nw, wl));
  CHECK_E(E, resident(buf, q, true, &d));
  char* dbase = d + bo[2] * bsp + bo[1] * brp + bo[0];
  char* hbase = ptr + ho[2] * hsp + ho[1] * hrp + ho[0];
  cl_int st = host_rect_copy(E, dbase, brp, bsp, hbase, hrp, hsp, region, write, blocking);
  if (st == CL_SUCCESS && write) written(buf, q);
  return st;
}

extern "C" cl_int clEnqueueReadBuffer(cl_command_queue q, cl_mem buf, cl_bool blocking,
                                      size_t offset, size_t size, void* ptr, cl_uint nw,
                                      const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, buf));
  if (size == 0 || offset > buf->size || size > buf->size - offset) return CL_INVALID_VALUE;
  const size_t bo[3] = {offset, 0, 0}, ho[3] = {0, 0, 0}, region[3] = {size, 1, 1};
  return buffer_host_rect(q, buf, blocking, bo, ho, region, 0, 0, 0, 0, static_cast<char*>(ptr),
                          false, nw, wl, ev, CL_COMMAND_READ_BUFFER);
}

extern "C" cl_int clEnqueueWriteBuffer(cl_command_queue q, cl_mem buf, cl_bool blocking,
                                       size_t offset, size_t size, const void* ptr, cl_uint nw,
                                       const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, buf));
  if (size == 0 || offset > buf->size || size > buf->size - offset) return CL_INVALID_VALUE;
  const size_t bo[3] = {offset, 0, 0}, ho[3] = {0, 0, 0}, region[3] = {size, 1, 1};
  return buffer_host_rect(q, buf, blocking, bo, ho, region, 0, 0, 0, 0,
                          const_cast<char*>(static_cast<const char*>(ptr)), true, nw, wl, ev,
                          CL_COMMAND_WRITE_BUFFER);
}

extern "C" cl_int clEnqueueReadBufferRect(cl_command_queue q, cl_mem buf, cl_bool blocking,
                                          const size_t* bo, const size_t* ho, const size_t* region,
                                          size_t brp, size_t bsp, size_t hrp, size_t hsp, void* ptr,
                                          cl_uint nw, const cl_event* wl, cl_event* ev) {
  return buffer_host_rect(q, buf, blocking, bo, ho, region, brp, bsp, hrp, hsp,
                          static_cast<char*>(ptr), false, nw, wl, ev, CL_COMMAND_READ_BUFFER_RECT);
}

extern "C" cl_int clEnqueueWriteBufferRect(cl_command_queue q, cl_mem buf, cl_bool blocking,
                                           const size_t* bo, const size_t* ho, const size_t* region,
                                           size_t brp, size_t bsp, size_t hrp, size_t hsp,
                                           const void* ptr, cl_uint nw, const cl_event* wl,
                                           cl_event* ev) {
  return buffer_host_rect(q, buf, blocking, bo, ho, region, brp, bsp, hrp, hsp,
                          const_cast<char*>(static_cast<const char*>(ptr)), true, nw, wl, ev,
                          CL_COMMAND_WRITE_BUFFER_RECT);
}

static cl_int image_host(cl_command_queue q, cl_mem img, cl_bool blocking, const size_t* origin,
                         const size_t* region, size_t rp, size_t sp, char* ptr, bool write,
                         cl_uint nw, const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, img));
  if (!is_image(img)) return CL_INVALID_MEM_OBJECT;
  const ImageLayout& L = img->img;
  if (!ptr) return CL_INVALID_VALUE;
  CHECK(validate_image_box(L.dims, L.w, L.h, L.d, origin, region));
  const size_t es = L.fmt.es;
  if (rp == 0) rp = region[0] * es;
  else if (rp < region[0] * es) return CL_INVALID_VALUE;
  if (L.arrayed && L.dims == 2) {
    // 1D image array: region[1] counts layers, host layers are slice_pitch
    // apart (0 -> row_pitch) ([CL1.2 §5.3.3]); they are the host's "rows"
    if (sp == 0) sp = rp;
    else if (sp < rp) return CL_INVALID_VALUE;
    rp = sp;
    sp = rp * region[1];
  } else {
    if (L.dims < 3 && sp != 0) return CL_INVALID_VALUE;
    if (sp == 0) sp = rp * region[1];
    else if (sp < rp * region[1]) return CL_INVALID_VALUE;
  }
  if (L.tiled) return tiled_image_host(q, img, blocking, origin, region, rp, sp, ptr, write, nw, wl, ev);
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = write ? CL_COMMAND_WRITE_IMAGE : CL_COMMAND_READ_IMAGE;
  DeviceGuard g(q->dev->ordinal);
  char* d = nullptr;
  CHECK(enq_begin(E, nw, wl));
  CHECK_E(E, resident(img, q, true, &d));
  char* dbase = d + origin[2] * L.slice_pitch + origin[1] * L.row_pitch + origin[0] * es;
  const size_t bytes_region[3] = {region[0] * es, region[1], region[2]};
  cl_int st = host_rect_copy(E, dbase, L.row_pitch, L.slice_pitch, ptr, rp, sp, bytes_region, write,
                             blocking);
  if (st == CL_SUCCESS && write) written(img, q);
  return st;
}

extern "C" cl_int clEnqueueReadImage(cl_command_queue q, cl_mem img, cl_bool blocking,
                                     const size_t* origin, const size_t* region, size_t rp,
                                     size_t sp, void* ptr, cl_uint nw, const cl_event* wl,
                                     cl_event* ev) {
  return image_host(q, img, blocking, origin, region, rp, sp, static_cast<char*>(ptr), false, nw,
                    wl, ev);
}

extern "C" cl_int clEnqueueWriteImage(cl_command_queue q, cl_mem img, cl_bool blocking,
                                      const size_t* origin, const size_t* region, size_t rp,
                                      size_t sp, const void* ptr, cl_uint nw, const cl_event* wl,
                                      cl_event* ev) {
  return image_host(q, img, blocking, origin, region, rp, sp,
                    const_cast<char*>(static_cast<const char*>(ptr)), true, nw, wl, ev);
}

// ===================================================================== device rect copies / fills
// One rect-copy kernel launch between two objects (already validated).
// The same box on the copy engines (the reference path of the
// b2clEnqueue*Engine extensions): cudaMemcpyAsync for one row,
// cudaMemcpy3DAsync when both slice pitches are whole rows, else one
// cudaMemcpy2DAsync per slice.
static cudaError_t engine_copy(const RectParams& p, cudaStream_t st) {
  if (p.R1 == 1 && p.R2 == 1) return cudaMemcpyAsync(p.dst, p.src, p.R0, cudaMemcpyDeviceToDevice, st);
  if (p.R2 == 1 || (p.ssp % p.srp == 0 && p.dsp % p.drp == 0)) {
    cudaMemcpy3DParms m{};
    m.srcPtr = make_cudaPitchedPtr(const_cast<char*>(p.src), p.srp, p.R0, p.R2 == 1 ? p.R1 : p.ssp / p.srp);
    m.dstPtr = make_cudaPitchedPtr(p.dst, p.drp, p.R0, p.R2 == 1 ? p.R1 : p.dsp / p.drp);
    m.extent = make_cudaExtent(p.R0, p.R1, p.R2);
    m.kind = cudaMemcpyDeviceToDevice;
    return cudaMemcpy3DAsync(&m, st);
  }
  cudaError_t e = cudaSuccess;
  for (uint32_t z = 0; z < p.R2 && e == cudaSuccess; ++z)
    e = cudaMemcpy2DAsync(p.dst + z * p.dsp, p.drp, p.src + z * p.ssp, p.srp, p.R0, p.R1, cudaMemcpyDeviceToDevice,
                          st);
  return e;
}

// copy_engine: the copy on the copy engines (engine_copy) instead of the SM
// kernel -- the reference path b2clEnqueueCopyBuffer{,Rect}Engine measure
static cl_int rect_copy(cl_command_queue q, cl_mem src, cl_mem dst, size_t soff, size_t doff,
                        const size_t* region_bytes, size_t srp, size_t ssp, size_t drp, size_t dsp,
                        cl_uint nw, const cl_event* wl, cl_event* ev, cl_command_type type,
                        bool copy_engine = false) {
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = type;
  DeviceGuard g(q->dev->ordinal);
  char *s = nullptr, *d = nullptr;
  Store* dst_store = nullptr;
  CHECK(enq_begin(E, nw, wl));
  CHECK_E(E, in_place(src, q, false, &s, nullptr));
  CHECK_E(E, in_place(dst, q, true, &d, &dst_store));
  RectParams p{};
  p.src = s + soff;
  p.dst = d + doff;
  p.R0 = region_bytes[0];
  p.R1 = (uint32_t)region_bytes[1];
  p.R2 = (uint32_t)region_bytes[2];
  p.srp = srp;
  p.ssp = ssp;
  p.drp = drp;
  p.dsp = dsp;
  cl_int st = enq_end(E, copy_engine ? engine_copy(p, q->stream) : launch_rect(p, RECT_COPY, q->stream));
  if (st == CL_SUCCESS) written_store(dst, dst_store);
  return st;
}

extern "C" cl_int clEnqueueCopyBufferRect(cl_command_queue q, cl_mem src, cl_mem dst,
                                          const size_t* so, const size_t* dso, const size_t* region,
                                          size_t srp, size_t ssp, size_t drp, size_t dsp, cl_uint nw,
                                          const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, src));
  CHECK(check_queue_mem(q, dst));
  if (src->type != CL_MEM_OBJECT_BUFFER || dst->type != CL_MEM_OBJECT_BUFFER)
    return CL_INVALID_MEM_OBJECT;
  CHECK(validate_copy_rect(src->size, dst->size, src == dst, so, dso, region, srp, ssp, drp, dsp));
  if (region[1] > 0xffffffffull || region[2] > 0xffffffffull) return CL_INVALID_VALUE;
  const size_t soff = so[2] * ssp + so[1] * srp + so[0];
  const size_t doff = dso[2] * dsp + dso[1] * drp + dso[0];
  return rect_copy(q, src, dst, soff, doff, region, srp, ssp, drp, dsp, nw, wl, ev,
                   CL_COMMAND_COPY_BUFFER_RECT);
}

extern "C" cl_int clEnqueueCopyBuffer(cl_command_queue q, cl_mem src, cl_mem dst, size_t so,
                                      size_t dso, size_t size, cl_uint nw, const cl_event* wl,
                                      cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, src));
  CHECK(check_queue_mem(q, dst));
  if (src->type != CL_MEM_OBJECT_BUFFER || dst->type != CL_MEM_OBJECT_BUFFER)
    return CL_INVALID_MEM_OBJECT;
  if (size == 0 || so > src->size || size > src->size - so || dso > dst->size ||
      size > dst->size - dso)
    return CL_INVALID_VALUE;
  if (src == dst && so < dso + size && dso < so + size) return CL_MEM_COPY_OVERLAP;
  const size_t region[3] = {size, 1, 1};
  return rect_copy(q, src, dst, so, dso, region, size, size, size, size, nw, wl, ev,
                   CL_COMMAND_COPY_BUFFER);
}

extern "C" cl_int clEnqueueFillBuffer(cl_command_queue q, cl_mem buf, const void* pattern,
                                      size_t ps, size_t offset, size_t size, cl_uint nw,
                                      const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, buf));
  if (buf->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_MEM_OBJECT;
  if (!pattern) return CL_INVALID_VALUE;
  CHECK(validate_fill_buffer(buf->size, ps, offset, size));
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = CL_COMMAND_FILL_BUFFER;
  DeviceGuard g(q->dev->ordinal);
  char* d = nullptr;
  Store* ds = nullptr;
  CHECK(enq_begin(E, nw, wl));
  CHECK_E(E, in_place(buf, q, true, &d, &ds));
  RectParams p{};
  p.dst = d + offset;
  p.R0 = size;
  p.R1 = p.R2 = 1;
  p.drp = p.dsp = size;
  // 128-byte tile indexed by absolute address: tile[X mod 128] = pattern[(X - start) mod ps]
  const uintptr_t start = reinterpret_cast<uintptr_t>(p.dst);
  unsigned char* tb = reinterpret_cast<unsigned char*>(p.ptile);
  const unsigned char* pat = static_cast<const unsigned char*>(pattern);
  for (uintptr_t k = 0; k < 128; ++k) tb[k] = pat[(k + 128 * ps - (start % ps)) % ps];
  cl_int st = enq_end(E, launch_rect(p, RECT_FILL, q->stream));
  if (st == CL_SUCCESS) written_store(buf, ds);
  return st;
}

static cl_int image_info_checked(cl_command_queue q, cl_mem m) {
  CHECK(check_queue_mem(q, m));
  if (!is_image(m)) return CL_INVALID_MEM_OBJECT;
  return CL_SUCCESS;
}

extern "C" cl_int clEnqueueCopyImage(cl_command_queue q, cl_mem src, cl_mem dst, const size_t* so,
                                     const size_t* dso, const size_t* region, cl_uint nw,
                                     const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(image_info_checked(q, src));
  CHECK(image_info_checked(q, dst));
  const ImageLayout &A = src->img, &B = dst->img;
  if (A.fmt.type != B.fmt.type || A.fmt.order != B.fmt.order) return CL_IMAGE_FORMAT_MISMATCH;
  CHECK(validate_image_box(A.dims, A.w, A.h, A.d, so, region));
  CHECK(validate_image_box(B.dims, B.w, B.h, B.d, dso, region));
  if (src == dst && image_boxes_overlap(so, dso, region)) return CL_MEM_COPY_OVERLAP;
  if (A.tiled || B.tiled) {
    return tex_enqueue(q, src, dst, [&](char* s, char* d, TexCopyParams& p) {
      p.src = image_side(src, s, so);
      p.dst = image_side(dst, d, dso);
      p.w = (uint32_t)region[0]; p.h = (uint32_t)region[1]; p.d = (uint32_t)region[2];
      p.es = (int)A.fmt.es;
    }, nw, wl, ev, CL_COMMAND_COPY_IMAGE);
  }
  const size_t es = A.fmt.es;
  const size_t soff = so[2] * A.slice_pitch + so[1] * A.row_pitch + so[0] * es;
  const size_t doff = dso[2] * B.slice_pitch + dso[1] * B.row_pitch + dso[0] * es;
  const size_t rb[3] = {region[0] * es, region[1], region[2]};
  return rect_copy(q, src, dst, soff, doff, rb, A.row_pitch, A.slice_pitch, B.row_pitch,
                   B.slice_pitch, nw, wl, ev, CL_COMMAND_COPY_IMAGE);
}

extern "C" cl_int clEnqueueCopyImageToBuffer(cl_command_queue q, cl_mem src, cl_mem dst,
                                             const size_t* so, const size_t* region, size_t doff,
                                             cl_uint nw, const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(image_info_checked(q, src));
  CHECK(check_queue_mem(q, dst));
  if (dst->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_MEM_OBJECT;
  const ImageLayout& A = src->img;
  CHECK(validate_image_box(A.dims, A.w, A.h, A.d, so, region));
  const size_t es = A.fmt.es, row = region[0] * es;
  const size_t bytes = row * region[1] * region[2];
  if (doff > dst->size || bytes > dst->size - doff) return CL_INVALID_VALUE;
  if (A.tiled) {
    return tex_enqueue(q, src, dst, [&](char* s, char* d, TexCopyParams& p) {
      p.src = image_side(src, s, so);
      p.dst = linear_side(d + doff, row, row * region[1]);
      p.w = (uint32_t)region[0]; p.h = (uint32_t)region[1]; p.d = (uint32_t)region[2];
      p.es = (int)es;
    }, nw, wl, ev, CL_COMMAND_COPY_IMAGE_TO_BUFFER);
  }
  const size_t soff = so[2] * A.slice_pitch + so[1] * A.row_pitch + so[0] * es;
  const size_t rb[3] = {row, region[1], region[2]};
  return rect_copy(q, src, dst, soff, doff, rb, A.row_pitch, A.slice_pitch, row, row * region[1],
                   nw, wl, ev, CL_COMMAND_COPY_IMAGE_TO_BUFFER);
}

extern "C" cl_int clEnqueueCopyBufferToImage(cl_command_queue q, cl_mem src, cl_mem dst,
                                             size_t soff, const size_t* dso, const size_t* region,
                                             cl_uint nw, const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, src));
  CHECK(image_info_checked(q, dst));
  if (src->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_MEM_OBJECT;
  const ImageLayout& B = dst->img;
  CHECK(validate_image_box(B.dims, B.w, B.h, B.d, dso, region));
  const size_t es = B.fmt.es, row = region[0] * es;
  const size_t bytes = row * region[1] * region[2];
  if (soff > src->size || bytes > src->size - soff) return CL_INVALID_VALUE;
  if (B.tiled) {
    return tex_enqueue(q, src, dst, [&](char* s, char* d, TexCopyParams& p) {
      p.src = linear_side(s + soff, row, row * region[1]);
      p.dst = image_side(dst, d, dso);
      p.w = (uint32_t)region[0]; p.h = (uint32_t)region[1]; p.d = (uint32_t)region[2];
      p.es = (int)es;
    }, nw, wl, ev, CL_COMMAND_COPY_BUFFER_TO_IMAGE);
  }
  const size_t doff = dso[2] * B.slice_pitch + dso[1] * B.row_pitch + dso[0] * es;
  const size_t rb[3] = {row, region[1], region[2]};
  return rect_copy(q, src, dst, soff, doff, rb, row, row * region[1], B.row_pitch, B.slice_pitch,
                   nw, wl, ev, CL_COMMAND_COPY_BUFFER_TO_IMAGE);
}

extern "C" cl_int clEnqueueFillImage(cl_command_queue q, cl_mem img, const void* color,
                                     const size_t* origin, const size_t* region, cl_uint nw,
                                     const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(image_info_checked(q, img));
  if (!color) return CL_INVALID_VALUE;
  const ImageLayout& L = img->img;
  CHECK(validate_image_box(L.dims, L.w, L.h, L.d, origin, region));
  if (L.tiled) {
    return tex_enqueue(q, nullptr, img, [&](char*, char* d, TexCopyParams& p) {
      p.dst = image_side(img, d, origin);
      p.w = (uint32_t)region[0]; p.h = (uint32_t)region[1]; p.d = (uint32_t)region[2];
      p.es = (int)L.fmt.es;
      p.fill = 1;
      memcpy(p.color, color, 16);
      p.type = L.fmt.type;
      p.order = L.fmt.order;
    }, nw, wl, ev, CL_COMMAND_FILL_IMAGE);
  }
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = CL_COMMAND_FILL_IMAGE;
  DeviceGuard g(q->dev->ordinal);
  char* d = nullptr;
  Store* ds = nullptr;
  CHECK(enq_begin(E, nw, wl));
  CHECK_E(E, in_place(img, q, true, &d, &ds));
  const size_t es = L.fmt.es;
  RectParams p{};
  p.dst = d + origin[2] * L.slice_pitch + origin[1] * L.row_pitch + origin[0] * es;
  p.R0 = region[0] * es;
  p.R1 = (uint32_t)region[1];
  p.R2 = (uint32_t)region[2];
  p.drp = L.row_pitch;
  p.dsp = L.slice_pitch;
  memcpy(p.color, color, 16);
  p.type = L.fmt.type;
  p.order = L.fmt.order;
  p.es = (int)es;
  cl_int st = enq_end(E, launch_rect(p, RECT_FILL_IMAGE, q->stream));
  if (st == CL_SUCCESS) written_store(img, ds);
  return st;
}

extern "C" cl_int clEnqueueMigrateMemObjects(cl_command_queue q, cl_uint n, const cl_mem* mems,
                                             cl_mem_migration_flags flags, cl_uint nw,
                                             const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  if (n == 0 || !mems) return CL_INVALID_VALUE;
  if (flags & ~(cl_mem_migration_flags)(CL_MIGRATE_MEM_OBJECT_HOST |
                                        CL_MIGRATE_MEM_OBJECT_CONTENT_UNDEFINED))
    return CL_INVALID_VALUE;
  for (cl_uint i = 0; i < n; ++i) CHECK(check_queue_mem(q, mems[i]));
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = CL_COMMAND_MIGRATE_MEM_OBJECTS;
  DeviceGuard g(q->dev->ordinal);
  CHECK(enq_begin(E, nw, wl));
  if (!(flags & CL_MIGRATE_MEM_OBJECT_HOST)) {  // HOST: device memory is the only storage (A24)
    const bool undefined = flags & CL_MIGRATE_MEM_OBJECT_CONTENT_UNDEFINED;
    for (cl_uint i = 0; i < n; ++i) {
      char* d = nullptr;
      CHECK_E(E, resident(mems[i], q, !undefined, &d));
      if (undefined) written(mems[i], q);  // ownership moves without a copy
    }
  }
  return enq_end(E, cudaSuccess);
}

extern "C" cl_int clEnqueueMarkerWithWaitList(cl_command_queue q, cl_uint nw, const cl_event* wl,
                                              cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = CL_COMMAND_MARKER;
  DeviceGuard g(q->dev->ordinal);
  CHECK(enq_begin(E, nw, wl));
  return enq_end(E, cudaSuccess);
}

extern "C" cl_int clEnqueueBarrierWithWaitList(cl_command_queue q, cl_uint nw, const cl_event* wl,
                                               cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = CL_COMMAND_BARRIER;
  DeviceGuard g(q->dev->ordinal);
  CHECK(enq_begin(E, nw, wl));
  return enq_end(E, cudaSuccess);
}

// ===================================================================== built-in extensions
static cl_int check_read_combo(cl_mem img, cl_sampler smp, b2cl_rtype rtype) {
  if (rtype > B2CL_RTYPE_UINT) return CL_INVALID_VALUE;
  if ((int)rtype != img->img.fmt.rclass) return CL_INVALID_OPERATION;           // A7
  if (rtype != B2CL_RTYPE_FLOAT && smp->filt == CL_FILTER_LINEAR) return CL_INVALID_OPERATION;  // A6
  return CL_SUCCESS;
}

static void fill_sampler(SampleParams& p, cl_sampler smp) {
  p.smp.norm = smp->norm ? 1 : 0;
  p.smp.addr = (int)(smp->addr - CL_ADDRESS_NONE);
  p.smp.filt = smp->filt == CL_FILTER_LINEAR ? dev::F_LINEAR : dev::F_NEAREST;
}

extern "C" cl_int b2clEnqueueReadImageSamples(cl_command_queue q, cl_mem img, cl_sampler smp,
                                              b2cl_rtype rtype, b2cl_ctype ctype, cl_mem coords,
                                              size_t coffset, size_t n, cl_mem out, size_t ooffset,
                                              cl_uint nw, const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(image_info_checked(q, img));
  if (!live(g_samplers, smp) || smp->ctx != q->ctx) return CL_INVALID_SAMPLER;
  CHECK(check_queue_mem(q, coords));
  CHECK(check_queue_mem(q, out));
  if (coords->type != CL_MEM_OBJECT_BUFFER || out->type != CL_MEM_OBJECT_BUFFER)
    return CL_INVALID_MEM_OBJECT;
  CHECK(check_read_combo(img, smp, rtype));
  if (ctype > B2CL_COORD_INT) return CL_INVALID_VALUE;
  if (ctype == B2CL_COORD_INT &&
      (smp->norm || smp->filt != CL_FILTER_NEAREST || smp->addr == CL_ADDRESS_REPEAT ||
       smp->addr == CL_ADDRESS_MIRRORED_REPEAT))
    return CL_INVALID_OPERATION;  // A30
  const int dims = img->img.dims;
  const size_t per = 4 * (dims == 1 ? 1 : (dims == 2 ? 2 : 4));
  if (coffset % per != 0 || ooffset % 16 != 0) return CL_INVALID_VALUE;
  if (n > 0 && (coffset > coords->size || n > (coords->size - coffset) / per ||
                ooffset > out->size || n > (out->size - ooffset) / 16))
    return CL_INVALID_VALUE;
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = 0x11F0;  // NDRANGE_KERNEL
  DeviceGuard g(q->dev->ordinal);
  char *pi = nullptr, *pc = nullptr, *po = nullptr;
  CHECK(enq_begin(E, nw, wl));
  CHECK_E(E, resident(img, q, true, &pi));
  CHECK_E(E, resident(coords, q, true, &pc));
  CHECK_E(E, resident(out, q, true, &po));
  SampleParams p{};
  p.im = dev_image(img, pi, true);
  fill_sampler(p, smp);
  p.rclass = (int)rtype;
  p.dims = dims - img->img.arrayed;  // sampled axes; an array's layer is coordinate p.dims
  p.arr = img->img.arrayed;
  p.coords = pc + coffset;
  p.n = n;
  p.out = po + ooffset;
  cl_int st = enq_end(E, launch_sample(p, ctype == B2CL_COORD_INT ? COORD_LIST_I : COORD_LIST_F,
                                       q->stream));
  if (st == CL_SUCCESS) written(out, q);
  return st;
}

extern "C" cl_int b2clEnqueueReadImageGridRegion(cl_command_queue q, cl_mem img, cl_sampler smp,
                                                 b2cl_rtype rtype, const float* affine,
                                                 const size_t* out_origin, const size_t* out_region,
                                                 cl_uint outc, cl_mem out, size_t ooffset,
                                                 cl_uint nw, const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(image_info_checked(q, img));
  if (!live(g_samplers, smp) || smp->ctx != q->ctx) return CL_INVALID_SAMPLER;
  CHECK(check_queue_mem(q, out));
  if (out->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_MEM_OBJECT;
  CHECK(check_read_combo(img, smp, rtype));
  if (!affine || !out_origin || !out_region || outc < 1 || outc > 4 || ooffset % 16 != 0)
    return CL_INVALID_VALUE;
  // output indices origin + [0, region) must be exact int32 -> float conversions' domain
  for (int k = 0; k < 3; ++k)
    if (out_origin[k] > 0x7fffffff || out_region[k] > 0x7fffffff - out_origin[k])
      return CL_INVALID_VALUE;
  if (out_region[2] > 65535) return CL_INVALID_VALUE;
  const unsigned __int128 bytes =
      (unsigned __int128)out_region[0] * out_region[1] * out_region[2] * outc * 4;
  if (ooffset > out->size || bytes > out->size - ooffset) return CL_INVALID_VALUE;
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = 0x11F0;
  DeviceGuard g(q->dev->ordinal);
  char *pi = nullptr, *po = nullptr;
  CHECK(enq_begin(E, nw, wl));
  CHECK_E(E, resident(img, q, true, &pi));
  CHECK_E(E, resident(out, q, true, &po));
  SampleParams p{};
  p.im = dev_image(img, pi, true);
  fill_sampler(p, smp);
  p.rclass = (int)rtype;
  p.dims = img->img.dims - img->img.arrayed;
  p.arr = img->img.arrayed;
  memcpy(p.A, affine, sizeof(p.A));
  p.ow = (int)out_region[0];
  p.oh = (int)out_region[1];
  p.od = (int)out_region[2];
  p.ox = (int)out_origin[0];
  p.oy = (int)out_origin[1];
  p.oz = (int)out_origin[2];
  p.outc = (int)outc;
  p.out = po + ooffset;
  cl_int st = enq_end(E, launch_sample(p, COORD_GRID, q->stream));
  if (st == CL_SUCCESS) written(out, q);
  return st;
}

extern "C" cl_int b2clEnqueueReadImageGrid(cl_command_queue q, cl_mem img, cl_sampler smp,
                                           b2cl_rtype rtype, const float* affine,
                                           const size_t* out_dims, cl_uint outc, cl_mem out,
                                           size_t ooffset, cl_uint nw, const cl_event* wl,
                                           cl_event* ev) {
  const size_t origin[3] = {0, 0, 0};
  return b2clEnqueueReadImageGridRegion(q, img, smp, rtype, affine, origin, out_dims, outc, out,
                                        ooffset, nw, wl, ev);
}

extern "C" cl_int b2clEnqueueWriteImageSamples(cl_command_queue q, cl_mem img, b2cl_rtype rtype,
                                               cl_mem coords, size_t coffset, size_t n,
                                               cl_mem colors, size_t koffset, cl_uint nw,
                                               const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(image_info_checked(q, img));
  CHECK(check_queue_mem(q, coords));
  CHECK(check_queue_mem(q, colors));
  if (coords->type != CL_MEM_OBJECT_BUFFER || colors->type != CL_MEM_OBJECT_BUFFER)
    return CL_INVALID_MEM_OBJECT;
  if (rtype > B2CL_RTYPE_UINT) return CL_INVALID_VALUE;
  if ((int)rtype != img->img.fmt.rclass) return CL_INVALID_OPERATION;  // A7
  const int dims = img->img.dims;
  const size_t per = 4 * (dims == 1 ? 1 : (dims == 2 ? 2 : 4));
  if (coffset % per != 0 || koffset % 16 != 0) return CL_INVALID_VALUE;
  if (n > 0 && (coffset > coords->size || n > (coords->size - coffset) / per ||
                koffset > colors->size || n > (colors->size - koffset) / 16))
    return CL_INVALID_VALUE;
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = 0x11F0;
  DeviceGuard g(q->dev->ordinal);
  char *pi = nullptr, *pc = nullptr, *pk = nullptr;
  CHECK(enq_begin(E, nw, wl));
  CHECK_E(E, resident(img, q, true, &pi));
  CHECK_E(E, resident(coords, q, true, &pc));
  CHECK_E(E, resident(colors, q, true, &pk));
  WriteParams p{};
  p.im = dev_image(img, pi);
  p.rclass = (int)rtype;
  p.dims = dims;
  p.coords = reinterpret_cast<const int32_t*>(pc + coffset);
  p.colors = reinterpret_cast<const uint32_t*>(pk + koffset);
  p.n = n;
  cl_int st = enq_end(E, launch_write(p, q->stream));
  if (st == CL_SUCCESS) written(img, q);
  return st;
}

// ===================================================================== interop
extern "C" cl_int b2clGetMemDevicePointer(cl_mem m, cl_device_id d, void** ptr) {
  if (!live(g_mems, m)) return CL_INVALID_MEM_OBJECT;
  if (!valid_device(d) || !ctx_has_device(m->ctx, d)) return CL_INVALID_DEVICE;
  if (!ptr) return CL_INVALID_VALUE;
  size_t off = 0;
  if (m->parent) {  // a 1D image buffer's (a view's) texels are its parent's
    off = m->parent_off;
    m = m->parent;
  }
  std::lock_guard<std::mutex> g(m->mu);
  Store* s = nullptr;
  CHECK(ensure_store(m, d->ordinal, nullptr, &s));
  *ptr = s->ptr + off;
  return CL_SUCCESS;
}

extern "C" cl_int b2clGetMemIpcHandle(cl_mem m, void* handle64) {
  if (!live(g_mems, m)) return CL_INVALID_MEM_OBJECT;
  if (!handle64) return CL_INVALID_VALUE;
  std::lock_guard<std::mutex> g(m->mu);
  if (!(m->flags & B2CL_MEM_IPC_EXPORTABLE) || m->stores.empty() || m->stores[0].kind != 1)
    return CL_INVALID_OPERATION;
  DeviceGuard dg(m->stores[0].ordinal);
  cudaIpcMemHandle_t h;
  cudaError_t e = cudaIpcGetMemHandle(&h, m->stores[0].ptr);
  if (e != cudaSuccess) return cuda_err(e);
  static_assert(sizeof(h) == 64, "IPC handle size");
  memcpy(handle64, &h, 64);
  return CL_SUCCESS;
}

extern "C" cl_mem b2clCreateBufferFromIpcHandle(cl_context c, cl_device_id d, const void* handle64,
                                                size_t size, cl_int* errcode_ret) {
  if (!live(g_contexts, c)) { SET_ERR(CL_INVALID_CONTEXT); return nullptr; }
  if (!valid_device(d) || !ctx_has_device(c, d)) { SET_ERR(CL_INVALID_DEVICE); return nullptr; }
  if (!handle64 || size == 0) { SET_ERR(CL_INVALID_VALUE); return nullptr; }
  cudaIpcMemHandle_t h;
  memcpy(&h, handle64, 64);
  void* p = nullptr;
  {
    DeviceGuard g(d->ordinal);
    cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) { SET_ERR(cuda_err(e)); return nullptr; }
  }
  cl_mem m = new_mem(c, CL_MEM_OBJECT_BUFFER, CL_MEM_READ_WRITE, size);
  if (!m) {
    DeviceGuard g(d->ordinal);
    cudaIpcCloseMemHandle(p);
    SET_ERR(CL_OUT_OF_HOST_MEMORY);
    return nullptr;
  }
  Store s;
  s.ordinal = d->ordinal;
  s.ptr = static_cast<char*>(p);
  s.kind = 4;  // another process's memory: its valid copy (kRemoteBit)
  m->stores.push_back(s);
  m->valid = 1ull << kRemoteBit;
  register_mem(m);
  SET_ERR(CL_SUCCESS);
  return m;
}

extern "C" cl_mem b2clCreateImageFromIpcHandle(cl_context c, cl_device_id d, cl_mem_flags flags,
                                               const cl_image_format* fmt, const cl_image_desc* desc,
                                               const void* handle64, cl_int* errcode_ret) {
  if (!live(g_contexts, c)) { SET_ERR(CL_INVALID_CONTEXT); return nullptr; }
  if (!valid_device(d) || !ctx_has_device(c, d)) { SET_ERR(CL_INVALID_DEVICE); return nullptr; }
  if (!handle64 || (flags & (CL_MEM_USE_HOST_PTR | CL_MEM_COPY_HOST_PTR | CL_MEM_ALLOC_HOST_PTR | B2CL_MEM_TILED_IMAGE))) {
    SET_ERR(CL_INVALID_VALUE);
    return nullptr;
  }
  ImageLayout L;
  cl_int st = image_layout(fmt, desc, &L);
  if (st != CL_SUCCESS) { SET_ERR(st); return nullptr; }
  if (desc->image_type == CL_MEM_OBJECT_IMAGE1D_BUFFER || desc->image_row_pitch || desc->image_slice_pitch) {
    SET_ERR(CL_INVALID_IMAGE_DESCRIPTOR);
    return nullptr;
  }
  cudaIpcMemHandle_t h;
  memcpy(&h, handle64, 64);
  void* p = nullptr;
  {
    DeviceGuard g(d->ordinal);
    cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) { SET_ERR(cuda_err(e)); return nullptr; }
  }
  cl_mem m = new_mem(c, desc->image_type, flags & (CL_MEM_READ_WRITE | CL_MEM_WRITE_ONLY | CL_MEM_READ_ONLY),
                     L.bytes);
  if (!m) {
    DeviceGuard g(d->ordinal);
    cudaIpcCloseMemHandle(p);
    SET_ERR(CL_OUT_OF_HOST_MEMORY);
    return nullptr;
  }
  m->img = L;
  m->fmt = *fmt;
  m->desc = *desc;
  Store s;
  s.ordinal = d->ordinal;
  s.ptr = static_cast<char*>(p);
  s.kind = 4;
  m->stores.push_back(s);
  m->valid = 1ull << kRemoteBit;
  register_mem(m);
  SET_ERR(CL_SUCCESS);
  return m;
}

extern "C" cl_int b2clEnqueueCopyBufferEngine(cl_command_queue q, cl_mem src, cl_mem dst, size_t so,
                                              size_t dso, size_t size, cl_uint nw, const cl_event* wl,
                                              cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, src));
  CHECK(check_queue_mem(q, dst));
  if (src->type != CL_MEM_OBJECT_BUFFER || dst->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_MEM_OBJECT;
  if (size == 0 || so > src->size || size > src->size - so || dso > dst->size || size > dst->size - dso)
    return CL_INVALID_VALUE;
  if (src == dst && so < dso + size && dso < so + size) return CL_MEM_COPY_OVERLAP;
  const size_t region[3] = {size, 1, 1};
  return rect_copy(q, src, dst, so, dso, region, size, size, size, size, nw, wl, ev, CL_COMMAND_COPY_BUFFER,
                   true);
}

extern "C" cl_int b2clEnqueueCopyBufferRectEngine(cl_command_queue q, cl_mem src, cl_mem dst, const size_t* so,
                                                  const size_t* dso, const size_t* region, size_t srp, size_t ssp,
                                                  size_t drp, size_t dsp, cl_uint nw, const cl_event* wl,
                                                  cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, src));
  CHECK(check_queue_mem(q, dst));
  if (src->type != CL_MEM_OBJECT_BUFFER || dst->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_MEM_OBJECT;
  CHECK(validate_copy_rect(src->size, dst->size, src == dst, so, dso, region, srp, ssp, drp, dsp));
  if (region[1] > 0xffffffffull || region[2] > 0xffffffffull) return CL_INVALID_VALUE;
  const size_t soff = so[2] * ssp + so[1] * srp + so[0];
  const size_t doff = dso[2] * dsp + dso[1] * drp + dso[0];
  return rect_copy(q, src, dst, soff, doff, region, srp, ssp, drp, dsp, nw, wl, ev, CL_COMMAND_COPY_BUFFER_RECT,
                   true);
}

extern "C" cl_int b2clEnqueueFillBufferEngine(cl_command_queue q, cl_mem buf, const void* pattern, size_t ps,
                                              size_t offset, size_t size, cl_uint nw, const cl_event* wl,
                                              cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  CHECK(check_queue_mem(q, buf));
  if (buf->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_MEM_OBJECT;
  if (!pattern || (ps != 1 && ps != 2 && ps != 4)) return CL_INVALID_VALUE;  // cuMemsetD8/16/32
  CHECK(validate_fill_buffer(buf->size, ps, offset, size));
  CHECK(check_wait_list(q, nw, wl));
  using memset_fn = CUresult (*)(CUdeviceptr, unsigned int, size_t, CUstream);
  static memset_fn fns[3] = {nullptr, nullptr, nullptr};
  static std::once_flag once;
  std::call_once(once, [] {
    const char* names[3] = {"cuMemsetD8Async", "cuMemsetD16Async", "cuMemsetD32Async"};
    for (int i = 0; i < 3; ++i) {
      void* f = nullptr;
      cudaDriverEntryPointQueryResult r;
      if (cudaGetDriverEntryPoint(names[i], &f, cudaEnableDefault, &r) == cudaSuccess &&
          r == cudaDriverEntryPointSuccess)
        fns[i] = reinterpret_cast<memset_fn>(f);
    }
  });
  const int which = ps == 1 ? 0 : (ps == 2 ? 1 : 2);
  if (!fns[which]) return CL_OUT_OF_RESOURCES;
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = CL_COMMAND_FILL_BUFFER;
  DeviceGuard g(q->dev->ordinal);
  char* d = nullptr;
  Store* ds = nullptr;
  CHECK(enq_begin(E, nw, wl));
  CHECK_E(E, in_place(buf, q, true, &d, &ds));
  unsigned int v = 0;
  memcpy(&v, pattern, ps);
  const CUresult r = fns[which](reinterpret_cast<CUdeviceptr>(d + offset), v, size / ps,
                                reinterpret_cast<CUstream>(q->stream));
  cl_int st = enq_end(E, r == CUDA_SUCCESS ? cudaSuccess : cudaErrorUnknown);
  if (st == CL_SUCCESS) written_store(buf, ds);
  return st;
}

// ===================================================================== programs and kernels
// The paper's OpenCL-to-CUDA launch path: clBuildProgram -> module load
// (P:119-121), clSetKernelArg collects the arguments, clEnqueueNDRangeKernel
// -> one launch with grid = global / local, __local arguments as
// sizes carving one dynamic shared array (Fig. 5(b)).
struct KArg {
  int kind = 0;  // 0 unset, 1 bytes, 2 memory object, 3 sampler, 4 __local, 5 __constant
  std::vector<unsigned char> bytes;
  cl_mem mem = nullptr;
  cl_sampler smp = nullptr;
  size_t local = 0;
};

struct _cl_program {
  std::atomic<int> ref{1};
  cl_context ctx;
  std::vector<int> ordinals;                        // one module per device
  std::vector<std::vector<unsigned char>> images;   // NUL-terminated (PTX text is allowed)
  std::vector<cudaLibrary_t> libs;
  std::vector<void*> offset_sym;                    // __b2cl_global_offset per module (or null)
  std::vector<void*> const_sym;                     // __OC2CU_const_mem per module (or null)
  size_t const_bytes = 0;
  std::mutex sym_mu;                                // orders launches that write the symbols
  std::vector<cudaEvent_t> sym_ev;                  // per module: the last such launch
  cl_int status = CL_BUILD_NONE;
  std::string log;
};

struct _cl_kernel {
  std::atomic<int> ref{1};
  cl_program prog;
  std::string name;
  std::vector<cudaKernel_t> kerns;  // per program module
  std::vector<size_t> psize;        // parameter sizes
  std::vector<KArg> args;
  uint32_t const_mask = 0;          // __constant arguments (B2CL_KERNEL_CONSTANT_ARGS)
};

static std::set<cl_program> g_programs;
static std::set<cl_kernel> g_kernels;

extern "C" cl_program clCreateProgramWithBinary(cl_context c, cl_uint n, const cl_device_id* devs,
                                                const size_t* lengths, const unsigned char** bins,
                                                cl_int* binary_status, cl_int* errcode_ret) {
  if (!live(g_contexts, c)) { SET_ERR(CL_INVALID_CONTEXT); return nullptr; }
  if (n == 0 || !devs || !lengths || !bins) { SET_ERR(CL_INVALID_VALUE); return nullptr; }
  auto* p = new (std::nothrow) _cl_program();
  if (!p) { SET_ERR(CL_OUT_OF_HOST_MEMORY); return nullptr; }
  p->ctx = c;
  for (cl_uint i = 0; i < n; ++i) {
    if (!valid_device(devs[i]) || !ctx_has_device(c, devs[i])) {
      delete p;
      SET_ERR(CL_INVALID_DEVICE);
      return nullptr;
    }
    if (lengths[i] == 0 || !bins[i]) {
      if (binary_status) binary_status[i] = CL_INVALID_VALUE;
      delete p;
      SET_ERR(CL_INVALID_VALUE);
      return nullptr;
    }
    if (binary_status) binary_status[i] = CL_SUCCESS;
    if (std::find(p->ordinals.begin(), p->ordinals.end(), devs[i]->ordinal) != p->ordinals.end())
      continue;
    p->ordinals.push_back(devs[i]->ordinal);
    std::vector<unsigned char> img(bins[i], bins[i] + lengths[i]);
    img.push_back(0);
    p->images.push_back(std::move(img));
  }
  c->ref++;
  {
    std::lock_guard<std::mutex> g(g_mu);
    g_programs.insert(p);
  }
  SET_ERR(CL_SUCCESS);
  return p;
}

extern "C" cl_int clBuildProgram(cl_program p, cl_uint n, const cl_device_id* devs,
                                 const char* options, void(CL_CALLBACK* notify)(cl_program, void*),
                                 void* user_data) {
  (void)options;
  if (!live(g_programs, p)) return CL_INVALID_PROGRAM;
  if ((n == 0) != (devs == nullptr) || (!notify && user_data)) return CL_INVALID_VALUE;
  if (!p->libs.empty()) return CL_INVALID_OPERATION;  // already built (kernels may exist)
  p->log.clear();
  for (size_t i = 0; i < p->ordinals.size(); ++i) {
    DeviceGuard g(p->ordinals[i]);
    cudaLibrary_t lib = nullptr;
    cudaError_t e = cudaLibraryLoadData(&lib, p->images[i].data(), nullptr, nullptr, 0, nullptr,
                                        nullptr, 0);
    // module loading may be lazy: an image with no kernel is a failed build
    unsigned nk = 0;
    if (e == cudaSuccess && (cudaLibraryGetKernelCount(&nk, lib) != cudaSuccess || nk == 0)) {
      cudaLibraryUnload(lib);
      e = cudaErrorInvalidKernelImage;
    }
    if (e != cudaSuccess) {
      cudaGetLastError();
      p->log = std::string("module load failed on device ") + std::to_string(p->ordinals[i]) +
               ": " + cudaGetErrorString(e);
      for (auto l : p->libs) cudaLibraryUnload(l);
      p->libs.clear();
      p->offset_sym.clear();
      p->const_sym.clear();
      p->sym_ev.clear();
      p->status = CL_BUILD_ERROR;
      if (notify) notify(p, user_data);
      return CL_BUILD_PROGRAM_FAILURE;
    }
    void* sym = nullptr;
    size_t bytes = 0;
    if (cudaLibraryGetGlobal(&sym, &bytes, lib, "__b2cl_global_offset") != cudaSuccess ||
        bytes < 3 * sizeof(size_t)) {
      cudaGetLastError();
      sym = nullptr;
    }
    void* csym = nullptr;
    size_t cbytes = 0;
    if (cudaLibraryGetGlobal(&csym, &cbytes, lib, "__OC2CU_const_mem") != cudaSuccess) {
      cudaGetLastError();
      csym = nullptr;
      cbytes = 0;
    }
    p->libs.push_back(lib);
    p->offset_sym.push_back(sym);
    p->const_sym.push_back(csym);
    p->sym_ev.push_back(nullptr);
    p->const_bytes = cbytes;
  }
  p->status = CL_BUILD_SUCCESS;
  if (notify) notify(p, user_data);
  return CL_SUCCESS;
}

extern "C" cl_int clGetProgramBuildInfo(cl_program p, cl_device_id d, cl_program_build_info name,
                                        size_t size, void* value, size_t* size_ret) {
  if (!live(g_programs, p)) return CL_INVALID_PROGRAM;
  if (!valid_device(d)) return CL_INVALID_DEVICE;
  switch (name) {
    case CL_PROGRAM_BUILD_STATUS: return get_info<cl_int>(p->status, size, value, size_ret);
    case CL_PROGRAM_BUILD_LOG: return get_str(p->log.c_str(), size, value, size_ret);
    default: return CL_INVALID_VALUE;
  }
}

extern "C" cl_int clRetainProgram(cl_program p) {
  return retain_ref(g_programs, p) ? CL_SUCCESS : CL_INVALID_PROGRAM;
}

extern "C" cl_int clReleaseProgram(cl_program p) {
  const int r = release_ref(g_programs, p);
  if (r < 0) return CL_INVALID_PROGRAM;
  if (r == 1) {
    for (size_t i = 0; i < p->libs.size(); ++i) {
      DeviceGuard g(p->ordinals[i]);
      cudaDeviceSynchronize();  // no launch of the module may still be running
      if (i < p->sym_ev.size() && p->sym_ev[i]) cudaEventDestroy(p->sym_ev[i]);
      cudaLibraryUnload(p->libs[i]);
    }
    cl_context c = p->ctx;
    delete p;
    clReleaseContext(c);
  }
  return CL_SUCCESS;
}

extern "C" cl_kernel clCreateKernel(cl_program p, const char* name, cl_int* errcode_ret) {
  if (!live(g_programs, p)) { SET_ERR(CL_INVALID_PROGRAM); return nullptr; }
  if (!name) { SET_ERR(CL_INVALID_VALUE); return nullptr; }
  if (p->status != CL_BUILD_SUCCESS) { SET_ERR(CL_INVALID_PROGRAM_EXECUTABLE); return nullptr; }
  auto* k = new (std::nothrow) _cl_kernel();
  if (!k) { SET_ERR(CL_OUT_OF_HOST_MEMORY); return nullptr; }
  k->prog = p;
  k->name = name;
  for (size_t i = 0; i < p->libs.size(); ++i) {
    DeviceGuard g(p->ordinals[i]);
    cudaKernel_t kern = nullptr;
    if (cudaLibraryGetKernel(&kern, p->libs[i], name) != cudaSuccess) {
      cudaGetLastError();
      delete k;
      SET_ERR(CL_INVALID_KERNEL_NAME);
      return nullptr;
    }
    k->kerns.push_back(kern);
  }
  // parameter sizes from the module's metadata
  {
    DeviceGuard g(p->ordinals[0]);
    for (size_t idx = 0;; ++idx) {
      size_t off = 0, sz = 0;
      if (cudaFuncGetParamInfo(reinterpret_cast<const void*>(k->kerns[0]), idx, &off, &sz) !=
          cudaSuccess) {
        cudaGetLastError();
        break;
      }
      k->psize.push_back(sz);
    }
  }
  k->args.resize(k->psize.size());
  {  // which arguments are __constant (a module global written by the translator)
    DeviceGuard g(p->ordinals[0]);
    void* m = nullptr;
    size_t mb = 0;
    const std::string sym = "__b2cl_const_args_" + k->name;
    if (cudaLibraryGetGlobal(&m, &mb, p->libs[0], sym.c_str()) == cudaSuccess && mb == 4) {
      if (cudaMemcpy(&k->const_mask, m, 4, cudaMemcpyDeviceToHost) != cudaSuccess) k->const_mask = 0;
    }
    cudaGetLastError();
  }
  p->ref++;
  {
    std::lock_guard<std::mutex> g(g_mu);
    g_kernels.insert(k);
  }
  SET_ERR(CL_SUCCESS);
  return k;
}

extern "C" cl_int clRetainKernel(cl_kernel k) {
  return retain_ref(g_kernels, k) ? CL_SUCCESS : CL_INVALID_KERNEL;
}

extern "C" cl_int clReleaseKernel(cl_kernel k) {
  const int r = release_ref(g_kernels, k);
  if (r < 0) return CL_INVALID_KERNEL;
  if (r == 1) {
    cl_program p = k->prog;
    delete k;
    clReleaseProgram(p);
  }
  return CL_SUCCESS;
}

extern "C" cl_int clGetKernelInfo(cl_kernel k, cl_kernel_info name, size_t size, void* value,
                                  size_t* size_ret) {
  if (!live(g_kernels, k)) return CL_INVALID_KERNEL;
  switch (name) {
    case CL_KERNEL_FUNCTION_NAME: return get_str(k->name.c_str(), size, value, size_ret);
    case CL_KERNEL_NUM_ARGS: return get_info<cl_uint>((cl_uint)k->psize.size(), size, value, size_ret);
    case CL_KERNEL_REFERENCE_COUNT: return get_info<cl_uint>(k->ref.load(), size, value, size_ret);
    default: return CL_INVALID_VALUE;
  }
}

extern "C" cl_int clSetKernelArg(cl_kernel k, cl_uint index, size_t size, const void* value) {
  if (!live(g_kernels, k)) return CL_INVALID_KERNEL;
  if (index >= k->psize.size()) return CL_INVALID_ARG_INDEX;
  const size_t want = k->psize[index];
  KArg a;
  const bool is_const = index < 32 && ((k->const_mask >> index) & 1u);
  if (is_const) {  // __constant buffer: the parameter is its size (Fig. 5(b))
    void* h = nullptr;
    if (value && size == sizeof(void*)) memcpy(&h, value, sizeof(void*));
    cl_mem m = static_cast<cl_mem>(h);
    if (!h || !live(g_mems, m) || m->type != CL_MEM_OBJECT_BUFFER) return CL_INVALID_ARG_VALUE;
    if (m->ctx != k->prog->ctx) return CL_INVALID_MEM_OBJECT;
    if (want != sizeof(size_t)) return CL_INVALID_ARG_SIZE;
    a.kind = 5;
    a.mem = m;
  } else if (!value) {  // __local: the kernel parameter is the size (Fig. 5(b))
    if (size == 0) return CL_INVALID_ARG_SIZE;
    if (want != sizeof(size_t)) return CL_INVALID_ARG_VALUE;
    a.kind = 4;
    a.local = size;
  } else {
    void* h = nullptr;
    if (size == sizeof(void*)) memcpy(&h, value, sizeof(void*));
    if (h && live(g_mems, static_cast<cl_mem>(h))) {
      cl_mem m = static_cast<cl_mem>(h);
      if (m->ctx != k->prog->ctx) return CL_INVALID_MEM_OBJECT;
      if (want != (is_image(m) ? sizeof(dev::Image) : sizeof(void*))) return CL_INVALID_ARG_SIZE;
      a.kind = 2;
      a.mem = m;
    } else if (h && live(g_samplers, static_cast<cl_sampler>(h))) {
      if (want != sizeof(uint32_t)) return CL_INVALID_ARG_SIZE;
      a.kind = 3;
      a.smp = static_cast<cl_sampler>(h);
    } else {
      if (size != want) return CL_INVALID_ARG_SIZE;
      a.kind = 1;
      a.bytes.assign(static_cast<const unsigned char*>(value),
                     static_cast<const unsigned char*>(value) + size);
    }
  }
  k->args[index] = std::move(a);
  return CL_SUCCESS;
}

// largest divisor of g not above cap
static size_t pick_local(size_t g, size_t cap) {
  for (size_t l = std::min(g, cap); l > 1; --l)
    if (g % l == 0) return l;
  return 1;
}

extern "C" cl_int clEnqueueNDRangeKernel(cl_command_queue q, cl_kernel k, cl_uint work_dim,
                                         const size_t* goff, const size_t* gws, const size_t* lws,
                                         cl_uint nw, const cl_event* wl, cl_event* ev) {
  if (!live(g_queues, q)) return CL_INVALID_COMMAND_QUEUE;
  if (!live(g_kernels, k)) return CL_INVALID_KERNEL;
  if (k->prog->ctx != q->ctx) return CL_INVALID_CONTEXT;
  const auto it = std::find(k->prog->ordinals.begin(), k->prog->ordinals.end(), q->dev->ordinal);
  if (it == k->prog->ordinals.end()) return CL_INVALID_PROGRAM_EXECUTABLE;
  const size_t mi = it - k->prog->ordinals.begin();
  if (work_dim < 1 || work_dim > 3) return CL_INVALID_WORK_DIMENSION;
  if (!gws) return CL_INVALID_VALUE;
  for (const KArg& a : k->args)
    if (a.kind == 0) return CL_INVALID_KERNEL_ARGS;
  size_t G[3] = {1, 1, 1}, Lw[3] = {1, 1, 1}, O[3] = {0, 0, 0};
  for (cl_uint d = 0; d < work_dim; ++d) {
    G[d] = gws[d];
    if (G[d] == 0) return -63;  // CL_INVALID_GLOBAL_WORK_SIZE
    if (goff) O[d] = goff[d];
  }
  if (lws) {
    for (cl_uint d = 0; d < work_dim; ++d) {
      Lw[d] = lws[d];
      if (Lw[d] == 0 || G[d] % Lw[d] != 0) return CL_INVALID_WORK_GROUP_SIZE;
    }
    if (Lw[0] > 1024 || Lw[1] > 1024 || Lw[2] > 64) return CL_INVALID_WORK_ITEM_SIZE;
    if (Lw[0] * Lw[1] * Lw[2] > 1024) return CL_INVALID_WORK_GROUP_SIZE;
  } else {
    const size_t caps[3][3] = {{256, 1, 1}, {32, 8, 1}, {32, 4, 2}};
    for (cl_uint d = 0; d < work_dim; ++d) Lw[d] = pick_local(G[d], caps[work_dim - 1][d]);
  }
  const size_t grid[3] = {G[0] / Lw[0], G[1] / Lw[1], G[2] / Lw[2]};
  if (grid[0] > 0x7fffffffull || grid[1] > 65535 || grid[2] > 65535) return -63;
  CHECK(check_wait_list(q, nw, wl));
  Enq E;
  E.q = q;
  E.evout = ev;
  E.type = CL_COMMAND_NDRANGE_KERNEL;
  DeviceGuard g(q->dev->ordinal);
  CHECK(enq_begin(E, nw, wl));  // the wait list first: argument migrations come after it
  // argument values, in parameter order
  const size_t na = k->args.size();
  std::vector<std::vector<unsigned char>> vals(na);
  std::vector<void*> argp(na);
  size_t local_bytes = 0, const_bytes = 0;
  for (const KArg& a : k->args)
    if (a.kind == 5) const_bytes += a.mem->size;
  if (const_bytes && (!k->prog->const_sym[mi] || const_bytes > k->prog->const_bytes))
    return enq_fail(E, CL_OUT_OF_RESOURCES);  // more __constant data than the module's constant array
  std::vector<std::pair<char*, size_t>> const_src;  // (device pointer, bytes) in argument order
  for (size_t i = 0; i < na; ++i) {
    const KArg& a = k->args[i];
    if (a.kind == 1) {
      vals[i] = a.bytes;
    } else if (a.kind == 2) {
      char* ptr = nullptr;
      CHECK_E(E, resident(a.mem, q, true, &ptr));
      if (is_image(a.mem)) {
        const dev::Image im = dev_image(a.mem, ptr, true);
        vals[i].resize(sizeof(im));
        memcpy(vals[i].data(), &im, sizeof(im));
      } else {
        vals[i].resize(sizeof(ptr));
        memcpy(vals[i].data(), &ptr, sizeof(ptr));
      }
    } else if (a.kind == 3) {
      const uint32_t bits = (a.smp->norm ? 1u : 0u) | ((a.smp->addr - CL_ADDRESS_NONE) << 1) |
                            (a.smp->filt == CL_FILTER_LINEAR ? 0x20u : 0x10u);
      vals[i].resize(4);
      memcpy(vals[i].data(), &bits, 4);
    } else if (a.kind == 5) {
      char* ptr = nullptr;
      CHECK_E(E, resident(a.mem, q, true, &ptr));
      const_src.emplace_back(ptr, a.mem->size);
      vals[i].resize(sizeof(size_t));
      memcpy(vals[i].data(), &a.mem->size, sizeof(size_t));
    } else {
      vals[i].resize(sizeof(size_t));
      memcpy(vals[i].data(), &a.local, sizeof(size_t));
      local_bytes += a.local;
    }
    argp[i] = vals[i].data();
  }
  const void* fn = reinterpret_cast<const void*>(k->kerns[mi]);
  cudaError_t e = cudaSuccess;
  if (local_bytes > 48 * 1024)
    e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)local_bytes);
  void* osym = k->prog->offset_sym[mi];
  // The global offset and the __constant array are module globals: a launch
  // on another queue must not overwrite them while this one still reads them.
  // Launches that use them are chained per module -- each waits for the
  // previous such launch's completion event (from any queue) before its copies.
  const bool uses_syms = osym || !const_src.empty();
  std::unique_lock<std::mutex> sym_lock(k->prog->sym_mu, std::defer_lock);
  if (uses_syms) {
    sym_lock.lock();
    if (e == cudaSuccess && k->prog->sym_ev[mi]) e = cudaStreamWaitEvent(q->stream, k->prog->sym_ev[mi], 0);
  }
  if (e == cudaSuccess && osym)  // get_global_offset(): pageable source, staged before return
    e = cudaMemcpyAsync(osym, O, sizeof(O), cudaMemcpyHostToDevice, q->stream);
  // deferred placement of __constant buffers: copied at launch
  size_t coff = 0;
  for (const auto& cs : const_src) {
    if (e != cudaSuccess) break;
    e = cudaMemcpyAsync(static_cast<char*>(k->prog->const_sym[mi]) + coff, cs.first, cs.second,
                        cudaMemcpyDeviceToDevice, q->stream);
    coff += cs.second;
  }
  if (e == cudaSuccess) {
    e = cudaLaunchKernel(fn, dim3((unsigned)grid[0], (unsigned)grid[1], (unsigned)grid[2]),
                         dim3((unsigned)Lw[0], (unsigned)Lw[1], (unsigned)Lw[2]), argp.data(),
                         local_bytes, q->stream);
    if (e == cudaSuccess) count_launch("user kernel (clEnqueueNDRangeKernel)");
  }
  if (uses_syms && e == cudaSuccess) {
    if (!k->prog->sym_ev[mi]) e = cudaEventCreateWithFlags(&k->prog->sym_ev[mi], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventRecord(k->prog->sym_ev[mi], q->stream);
  }
  if (uses_syms) sym_lock.unlock();
  cl_int st = enq_end(E, e);
  if (st == CL_SUCCESS)
    for (const KArg& a : k->args)
      if (a.kind == 2) written(a.mem, q);  // __constant (kind 5) buffers are only read
  return st;
}

extern "C" cl_ulong b2clGetKernelLaunchCount(void) { return launch_count(); }

extern "C" const char* b2clGetLastKernelName(void) { return last_kernel(); }
