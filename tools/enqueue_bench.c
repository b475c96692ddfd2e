/* enqueue_bench.c -- host cost of one enqueue through the C-ABI, measured
 * from C (no Python / ctypes in the loop).
 *
 *   gcc -O2 -o build/enqueue_bench tools/enqueue_bench.c -ldl && build/enqueue_bench [libb2cl.so]
 *
 * For each call: N back-to-back enqueues timed with the host clock
 * (CLOCK_MONOTONIC) between a clFinish before and the return of the last
 * call (the GPU work is tiny and runs behind the host, so the time is the
 * host's), reported as microseconds per call; then a clFinish.  Calls:
 *   clEnqueueCopyImageToBuffer   4 KiB (a 256-texel RGBA32F image row)
 *   b2clEnqueueReadImageGrid     a 16 x 16 grid of a 64 x 64 RGBA32F image
 *   clEnqueueFillBuffer          4 KiB
 *   clEnqueueMarkerWithWaitList  (no kernel: the runtime's own overhead)
 * Prints one JSON object.  Needs a GPU; the library is loaded with dlopen. */
#define _GNU_SOURCE
#include <dlfcn.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

typedef int32_t cl_int;
typedef uint32_t cl_uint;
typedef uint64_t cl_ulong;
typedef void* H;
typedef struct { cl_uint order, type; } fmt_t;
typedef struct {
  cl_uint image_type;
  size_t w, h, d, array_size, row_pitch, slice_pitch;
  cl_uint mips, samples;
  H buffer;
} desc_t;

#define LOAD(name, ret, ...)                      \
  typedef ret (*name##_t)(__VA_ARGS__);           \
  name##_t name = (name##_t)dlsym(lib, #name);    \
  if (!name) { fprintf(stderr, "missing %s\n", #name); return 2; }

static double now_us(void) {
  struct timespec t;
  clock_gettime(CLOCK_MONOTONIC, &t);
  return t.tv_sec * 1e6 + t.tv_nsec * 1e-3;
}

int main(int argc, char** argv) {
  const char* path = argc > 1 ? argv[1] : "paper_conf_sc_kimdjjl15_b200/libb2cl.so";
  void* lib = dlopen(path, RTLD_NOW);
  if (!lib) { fprintf(stderr, "%s\n", dlerror()); return 2; }
  LOAD(clGetPlatformIDs, cl_int, cl_uint, H*, cl_uint*);
  LOAD(clGetDeviceIDs, cl_int, H, cl_ulong, cl_uint, H*, cl_uint*);
  LOAD(clCreateContext, H, const intptr_t*, cl_uint, const H*, void*, void*, cl_int*);
  LOAD(clCreateCommandQueue, H, H, H, cl_ulong, cl_int*);
  LOAD(clCreateBuffer, H, H, cl_ulong, size_t, void*, cl_int*);
  LOAD(clCreateImage, H, H, cl_ulong, const fmt_t*, const desc_t*, void*, cl_int*);
  LOAD(clCreateSampler, H, H, cl_uint, cl_uint, cl_uint, cl_int*);
  LOAD(clFinish, cl_int, H);
  LOAD(clEnqueueCopyImageToBuffer, cl_int, H, H, H, const size_t*, const size_t*, size_t, cl_uint, const H*, H*);
  LOAD(b2clEnqueueReadImageGrid, cl_int, H, H, H, cl_uint, const float*, const size_t*, cl_uint, H, size_t,
       cl_uint, const H*, H*);
  LOAD(clEnqueueFillBuffer, cl_int, H, H, const void*, size_t, size_t, size_t, cl_uint, const H*, H*);
  LOAD(clEnqueueMarkerWithWaitList, cl_int, H, cl_uint, const H*, H*);
  LOAD(clReleaseEvent, cl_int, H);
  H plat, dev;
  cl_int err = 0;
  if (clGetPlatformIDs(1, &plat, NULL) || clGetDeviceIDs(plat, 4 /*GPU*/, 1, &dev, NULL)) return 3;
  H ctx = clCreateContext(NULL, 1, &dev, NULL, NULL, &err);
  H q = clCreateCommandQueue(ctx, dev, 0, &err);
  fmt_t f = {0x10B5 /*RGBA*/, 0x10DE /*FLOAT*/};
  desc_t d1 = {0x10F1 /*IMAGE2D*/, 256, 1, 0, 0, 0, 0, 0, 0, NULL};
  desc_t d2 = {0x10F1, 64, 64, 0, 0, 0, 0, 0, 0, NULL};
  H img1 = clCreateImage(ctx, 1, &f, &d1, NULL, &err);
  H img2 = clCreateImage(ctx, 1, &f, &d2, NULL, &err);
  H buf = clCreateBuffer(ctx, 1, 1 << 16, NULL, &err);
  H smp = clCreateSampler(ctx, 1, 0x1133 /*REPEAT*/, 0x1141 /*LINEAR*/, &err);
  if (err) { fprintf(stderr, "setup failed %d\n", err); return 4; }
  const size_t zero[3] = {0, 0, 0}, r1[3] = {256, 1, 1}, gdim[3] = {16, 16, 1};
  const float A[12] = {1.f / 16, 0, 0, 0.01f, 0, 1.f / 16, 0, 0.02f, 0, 0, 0, 0};
  const unsigned char pat[16] = {1, 2, 3, 4, 5, 6, 7, 8, 9, 10, 11, 12, 13, 14, 15, 16};
  enum { N = 2000 };
  double us[4];
  for (int which = 0; which < 4; ++which) {
    for (int pass = 0; pass < 2; ++pass) {  // pass 0: warm-up
      clFinish(q);
      const double t0 = now_us();
      for (int i = 0; i < N; ++i) {
        cl_int st = 0;
        H ev = NULL;
        switch (which) {
          case 0: st = clEnqueueCopyImageToBuffer(q, img1, buf, zero, r1, 0, 0, NULL, NULL); break;
          case 1: st = b2clEnqueueReadImageGrid(q, img2, smp, 0, A, gdim, 4, buf, 0, 0, NULL, NULL); break;
          case 2: st = clEnqueueFillBuffer(q, buf, pat, 16, 0, 4096, 0, NULL, NULL); break;
          default:
            st = clEnqueueMarkerWithWaitList(q, 0, NULL, &ev);
            clReleaseEvent(ev);
            break;
        }
        if (st) { fprintf(stderr, "call %d failed %d\n", which, st); return 5; }
      }
      us[which] = (now_us() - t0) / N;
      clFinish(q);
    }
  }
  printf("{\"copy_image_to_buffer_4KiB_us\": %.3f, \"read_image_grid_16x16_us\": %.3f, "
         "\"fill_buffer_4KiB_us\": %.3f, \"marker_with_event_us\": %.3f, \"calls\": %d}\n",
         us[0], us[1], us[2], us[3], N);
  return 0;
}
