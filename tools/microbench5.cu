// microbench5.cu -- cost of one cooperative-groups grid barrier on B200, and of
// scanning a 24M-slot frontier bitmap (3 MB, L2-resident) per iteration, as a
// function of the grid size (the persistent SSSP loop's fixed cost per iteration).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/microbench5 tools/microbench5.cu
#include <cooperative_groups.h>
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

__global__ void k_sync(int iters, unsigned* sink) {
  cg::grid_group g = cg::this_grid();
  for (int i = 0; i < iters; i++) g.sync();
  if (threadIdx.x == 0 && blockIdx.x == 0) sink[0] = iters;
}

__global__ void k_scan_sync(const uint32_t* bm, int64_t nwords, int iters, unsigned* sink) {
  cg::grid_group g = cg::this_grid();
  unsigned acc = 0;
  for (int i = 0; i < iters; i++) {
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < nwords; w += (int64_t)gridDim.x * blockDim.x)
      acc += __ldcg(bm + w);
    g.sync();
  }
  if (acc == 12345) sink[1] = acc;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned* sink;
  uint32_t* bm;
  const int64_t nwords = 750000;
  cudaMalloc(&sink, 16);
  cudaMalloc(&bm, nwords * 4);
  cudaMemset(bm, 0, nwords * 4);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int per : {1, 2, 4}) {
    for (int thr : {256, 512, 1024}) {
      if (per * thr > 2048) continue;
      int grid = sms * per, iters = 2000;
      void* a1[] = {&iters, &sink};
      cudaLaunchCooperativeKernel((void*)k_sync, grid, thr, a1, 0, 0);
      cudaEventRecord(e0);
      cudaLaunchCooperativeKernel((void*)k_sync, grid, thr, a1, 0, 0);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      float us_sync = 1e3f * ms / iters;
      void* a2[] = {&bm, (void*)&nwords, &iters, &sink};
      cudaLaunchCooperativeKernel((void*)k_scan_sync, grid, thr, a2, 0, 0);
      cudaEventRecord(e0);
      cudaLaunchCooperativeKernel((void*)k_scan_sync, grid, thr, a2, 0, 0);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      cudaEventElapsedTime(&ms, e0, e1);
      printf("grid %4d x %4d threads: grid.sync %.2f us   scan 3 MB + sync %.2f us   %s\n", grid, thr, us_sync,
             1e3f * ms / iters, cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
