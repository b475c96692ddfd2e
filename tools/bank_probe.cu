// bank_probe.cu -- shared-memory wavefronts of given warp address patterns
// (A/B tool for the rotated-map kernel's box pitch; read with ncu:
//  l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum / requests).
//   nvcc -gencode arch=compute_100a,code=sm_100a -o build/bank_probe tools/bank_probe.cu
//   build/bank_probe patterns.bin     (int32 word addresses, 32 per pattern)
#include <cstdio>
#include <cstdlib>
#include <vector>

__global__ void probe(const int* addr, int npat, float* sink) {
  __shared__ float sm[12000];
  for (int i = threadIdx.x; i < 12000; i += blockDim.x) sm[i] = (float)i;
  __syncthreads();
  float acc = 0.f;
  for (int p = 0; p < npat; ++p) {
    const int a = addr[p * 32 + threadIdx.x];
    float v;
    asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"((unsigned)(__cvta_generic_to_shared(sm + a))));
    acc += v;
  }
  sink[threadIdx.x] = acc;
}

int main(int argc, char** argv) {
  FILE* f = fopen(argv[1], "rb");
  if (!f) return 2;
  std::vector<int> h;
  int x;
  while (fread(&x, 4, 1, f) == 1) h.push_back(x);
  fclose(f);
  const int npat = (int)h.size() / 32;
  int* d;
  float* s;
  cudaMalloc(&d, h.size() * 4);
  cudaMalloc(&s, 128);
  cudaMemcpy(d, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  probe<<<1, 32>>>(d, npat, s);
  cudaDeviceSynchronize();
  printf("%d patterns\n", npat);
  return 0;
}
