// Microbenchmark: HBM write rate of an n x n fp32 matrix written in tiles of TR rows x TC
// columns per CTA (persistent grid, contiguous row-major tile ranges per CTA, streaming
// st.global.cs.v4, each warp instruction = 512 contiguous bytes of one row). Question it
// answers: does the hd2 epilogue's tile shape (128 x 256 per CTA) limit the write rate that
// the d = 3 Type-III kernel (16 rows x full width) reaches?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/write_pattern tools/write_pattern.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void __launch_bounds__(512) tiles(float* out, int n, int TR, int TC, int raster) {
  const long long tj = n / TC, ti = n / TR, nt = ti * tj;
  // raster 0/1: a contiguous range of tiles per CTA (row- / column-major); 2: row-major tiles
  // dealt round-robin over CTAs (the tiles in flight are adjacent in memory)
  const bool rr = raster == 2;
  const long long b = rr ? blockIdx.x : nt * blockIdx.x / gridDim.x;
  const long long e = rr ? nt : nt * (blockIdx.x + 1) / gridDim.x;
  const long long step = rr ? gridDim.x : 1;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  const float4 v = make_float4(1.f, 2.f, 3.f, 4.f);
  for (long long t = b; t < e; t += step) {
    long long I, J;
    if (raster != 1) { I = t / tj; J = t % tj; }         // row-major tiles
    else { I = t % ti; J = t / ti; }                    // column-major tiles
    float* base = out + (size_t)I * TR * n + (size_t)J * TC;
    for (int r = warp; r < TR; r += nw)
      for (int c = lane * 4; c < TC; c += 128) __stcs(reinterpret_cast<float4*>(base + (size_t)r * n + c), v);
  }
}

// The d = 3 Type-III kernel's launch shape: one non-persistent CTA per (1024-column block,
// 16-row block), blockIdx.x over columns; each thread writes 4 columns of 16 rows.
__global__ void __launch_bounds__(256) grid2d(float* out, int n, int rows) {
  const int j0 = blockIdx.x * 1024 + threadIdx.x * 4;
  const float4 v = make_float4(1.f, 2.f, 3.f, 4.f);
  for (int i = blockIdx.y * rows; i < (blockIdx.y + 1) * rows; ++i)
    __stcs(reinterpret_cast<float4*>(out + (size_t)i * n + j0), v);
}
// The same with blockIdx.x over row blocks (tiles in flight far apart in memory).
__global__ void __launch_bounds__(256) grid2d_t(float* out, int n, int rows) {
  const int j0 = blockIdx.y * 1024 + threadIdx.x * 4;
  const float4 v = make_float4(1.f, 2.f, 3.f, 4.f);
  for (int i = blockIdx.x * rows; i < (blockIdx.x + 1) * rows; ++i)
    __stcs(reinterpret_cast<float4*>(out + (size_t)i * n + j0), v);
}

int main() {
  const int n = 65536;
  float* out;
  cudaMalloc(&out, (size_t)n * n * 4);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  struct { int TR, TC, raster, grid_mult, threads; } cfgs[] = {
      {128, 256, 0, 1, 512}, {128, 256, 1, 1, 512}, {256, 256, 0, 1, 512}, {128, 512, 0, 1, 512},
      {128, 1024, 0, 1, 512}, {64, 1024, 0, 1, 512}, {16, 1024, 0, 1, 256}, {16, 1024, 0, 4, 256},
      {16, 4096, 0, 1, 512}, {128, 256, 0, 2, 512}, {32, 256, 0, 1, 512},
      {128, 256, 2, 1, 512}, {128, 512, 2, 1, 512}, {16, 1024, 2, 1, 256}, {16, 1024, 2, 4, 256}, {128, 256, 2, 2, 512}};
  for (auto& c : cfgs) {
    const int grid = sms * c.grid_mult;
    for (int w = 0; w < 2; ++w) tiles<<<grid, c.threads>>>(out, n, c.TR, c.TC, c.raster);
    cudaEventRecord(a);
    const int reps = 5;
    for (int r = 0; r < reps; ++r) tiles<<<grid, c.threads>>>(out, n, c.TR, c.TC, c.raster);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    ms /= reps;
    printf("{\"TR\": %d, \"TC\": %d, \"raster\": \"%s\", \"grid\": %d, \"threads\": %d, \"ms\": %.4f, \"TBps\": %.3f}\n", c.TR, c.TC,
           c.raster == 2 ? "row-rr" : c.raster ? "col" : "row", grid, c.threads, ms, (double)n * n * 4 / ms / 1e9);
  }
  for (int rows : {16, 64, 128}) {
    for (int tr = 0; tr < 2; ++tr) {
      dim3 g = tr ? dim3(n / rows, n / 1024) : dim3(n / 1024, n / rows);
      for (int w = 0; w < 2; ++w) (tr ? grid2d_t : grid2d)<<<g, 256>>>(out, n, rows);
      cudaEventRecord(a);
      for (int r = 0; r < 5; ++r) (tr ? grid2d_t : grid2d)<<<g, 256>>>(out, n, rows);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      ms /= 5;
      printf("{\"grid2d\": \"%s\", \"rows\": %d, \"ms\": %.4f, \"TBps\": %.3f}\n", tr ? "rows-fast" : "cols-fast", rows, ms,
             (double)n * n * 4 / ms / 1e9);
    }
  }
  cudaEventRecord(a);
  for (int r = 0; r < 5; ++r) cudaMemsetAsync(out, 0, (size_t)n * n * 4);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  {
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    ms /= 5;
    printf("{\"memset\": true, \"ms\": %.4f, \"TBps\": %.3f}\n", ms, (double)n * n * 4 / ms / 1e9);
  }
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
