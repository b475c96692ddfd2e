// mix_probe.cu -- what HBM delivers for a streaming kernel with the C2
// MIRRORED pass's traffic mix (67 MB read, 268 MB written: 1 : 4), against a
// plain copy (1 : 1) and a pure write, so the fold kernel's time can be read
// against the floor of its own read/write mix rather than the copy peak.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mix_probe tools/mix_probe.cu && /tmp/mix_probe
#include <cstdio>
#include <cuda_runtime.h>

// each thread: U rounds of (R float4 reads, W float4 streaming writes), all
// coalesced: read r of element i at src[r * n + i], write w at dst[w * n + i]
// (the fold writes four mirror tiles: four write streams)
template <int R, int W, int U>
__global__ void __launch_bounds__(256) k_mix(const float4* __restrict__ src, float4* __restrict__ dst, long n) {
  const long stride = (long)gridDim.x * blockDim.x;
  for (long i0 = blockIdx.x * (long)blockDim.x + threadIdx.x; i0 < n; i0 += stride * U) {
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      v[u] = make_float4(0.f, 0.f, 0.f, 0.f);
      const long i = i0 + u * stride;
#pragma unroll
      for (int r = 0; r < R; ++r)
        if (i < n) {
          const float4 t = __ldcs(src + (long)r * n + i);
          v[u].x += t.x; v[u].y += t.y; v[u].z += t.z; v[u].w += t.w;
        }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const long i = i0 + u * stride;
      if (i < n)
#pragma unroll
        for (int w = 0; w < W; ++w) __stcs(dst + (long)w * n + i, make_float4(v[u].x + w, v[u].y, v[u].z, v[u].w));
    }
  }
}

template <int R, int W, int U>
static void run(const char* name, const float4* src, float4* dst, long n, int blocks) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int i = 0; i < 3; ++i) k_mix<R, W, U><<<blocks, 256>>>(src, dst, n);
  const int it = 20;
  cudaEventRecord(e0);
  for (int i = 0; i < it; ++i) k_mix<R, W, U><<<blocks, 256>>>(src, dst, n);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms = 0.f;
  cudaEventElapsedTime(&ms, e0, e1);
  const double us = ms * 1e3 / it;
  const double rd = (double)n * R * 16, wr = (double)n * W * 16;
  printf("%-34s read %6.1f MB write %6.1f MB  %7.1f us  %7.1f GB/s\n", name, rd / 1e6, wr / 1e6, us,
         (rd + wr) / us / 1e3);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
}

int main() {
  const long texels = 4096L * 4096 / 4;  // the folded quarter: 4.19 M RGBA32F texels (67 MB)
  float4 *src, *dst;
  cudaMalloc(&src, texels * 4 * 16);
  cudaMalloc(&dst, texels * 4 * 16);
  cudaMemset(src, 0, texels * 4 * 16);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int bps : {2, 4, 8, 16}) {
    const int blocks = sms * bps;
    printf("-- %d blocks of 256 threads\n", blocks);
    run<1, 4, 1>("1:4 (fold mix), 1 in flight", src, dst, texels, blocks);
    run<1, 4, 4>("1:4 (fold mix), 4 in flight", src, dst, texels, blocks);
    run<1, 1, 4>("1:1 copy, 268 MB each way", src, dst, texels * 4, blocks);
    run<0, 4, 4>("write only, 268 MB", src, dst, texels, blocks);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) printf("error %s\n", cudaGetErrorString(e));
  return e == cudaSuccess ? 0 : 1;
}
