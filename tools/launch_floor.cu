// launch_floor.cu -- the CUDA runtime's own host cost of one kernel launch on
// this box (the floor under any enqueue call of libb2cl):
//   nvcc -O2 -gencode arch=compute_100a,code=sm_100a -o build/launch_floor tools/launch_floor.cu
// Times 2000 back-to-back launches of an empty kernel taking a P-byte
// parameter block (P = 64, 256, 512: SampleParams / RectParams are ~200-300 B)
// with the host clock; prints JSON.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdio.h>
#include <time.h>

template <int P>
struct Blob { unsigned char b[P]; };

template <int P>
__global__ void empty_kernel(const Blob<P> p) {
  if (p.b[0] == 123 && threadIdx.x == 9999) printf("x");
}

static double now_us() {
  timespec t;
  clock_gettime(CLOCK_MONOTONIC, &t);
  return t.tv_sec * 1e6 + t.tv_nsec * 1e-3;
}

template <int P>
static double run(cudaStream_t s) {
  Blob<P> b = {};
  for (int pass = 0; pass < 2; ++pass) {
    cudaStreamSynchronize(s);
    const double t0 = now_us();
    for (int i = 0; i < 2000; ++i) empty_kernel<P><<<1, 32, 0, s>>>(b);
    const double dt = (now_us() - t0) / 2000;
    cudaStreamSynchronize(s);
    if (pass) return dt;
  }
  return 0;
}

// the driver API entry (cuLaunchKernel) with the CUfunction looked up once
template <int P>
static double run_driver(cudaStream_t s) {
  Blob<P> b = {};
  CUfunction f;
  cudaGetFuncBySymbol(&f, reinterpret_cast<const void*>(empty_kernel<P>));
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuLaunchKernel", &fn, cudaEnableDefault, &q);
  auto launch = reinterpret_cast<CUresult (*)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                                              unsigned, CUstream, void**, void**)>(fn);
  void* args[1] = {&b};
  for (int pass = 0; pass < 2; ++pass) {
    cudaStreamSynchronize(s);
    const double t0 = now_us();
    for (int i = 0; i < 2000; ++i) launch(f, 1, 1, 1, 32, 1, 1, 0, (CUstream)s, args, nullptr);
    const double dt = (now_us() - t0) / 2000;
    cudaStreamSynchronize(s);
    if (pass) return dt;
  }
  return 0;
}

int main() {
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  const double a = run<64>(s), b = run<256>(s), c = run<512>(s);
  int d = 0;
  cudaGetDevice(&d);
  double g0 = now_us();
  for (int i = 0; i < 10000; ++i) cudaGetDevice(&d);
  const double gd = (now_us() - g0) / 10000;
  const double da = run_driver<64>(s), db = run_driver<256>(s);
  printf("{\"launch_us_64B\": %.3f, \"launch_us_256B\": %.3f, \"launch_us_512B\": %.3f, \"cudaGetDevice_us\": %.4f, "
         "\"cuLaunchKernel_us_64B\": %.3f, \"cuLaunchKernel_us_256B\": %.3f}\n",
         a, b, c, gd, da, db);
  return 0;
}
