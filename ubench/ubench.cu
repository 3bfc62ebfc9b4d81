// Roofline micro-benchmarks for the denominators MEASURED_PEAKS.json lacks
// (SURVEY.md §7 step 0, §8(d) "Roofline denominators"): per-SM issue rate of the
// integer max-plus instructions the DP kernels use (VIADDMNMX s32 / s16x2,
// VIMNMX3), FFMA, LDS.128 bandwidth, and __syncthreads / grid-sync latency.
//
// Each kernel runs one 1024-thread CTA per SM (148 CTAs), 8 independent
// dependency chains per thread, and records clock64() around the timed loop.
// Result = lane-ops per SM clock (an s16x2 instruction counts as 2 lane-ops).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ubench ubench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <cooperative_groups.h>
namespace cg = cooperative_groups;

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); return 1; } } while (0)

constexpr int ITERS = 4096;
constexpr int CH = 8;

template <int OP>
__global__ void __launch_bounds__(1024, 1) k_alu(const int* in, int* out, long long* cyc) {
  int a[CH], b = in[threadIdx.x & 7] | 1, c = in[(threadIdx.x + 3) & 7];
  for (int q = 0; q < CH; ++q) a[q] = in[q] + threadIdx.x;
  __syncthreads();
  long long t0 = clock64();
#pragma unroll 4
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int q = 0; q < CH; ++q) {
      if (OP == 0) a[q] = __viaddmax_s32(a[q], b, c);
      if (OP == 1) a[q] = (int)__viaddmax_s16x2((unsigned)a[q], (unsigned)b, (unsigned)c);
      if (OP == 2) a[q] = __vimax3_s32(a[q], b, c);
      if (OP == 3) a[q] = (int)__vimax3_s16x2_relu((unsigned)a[q], (unsigned)b, (unsigned)c);
      // plain IMNMX / IADD chains in volatile asm: a C++ max(a, b) or a + b chain is folded by
      // the compiler (round 1's rows of 7.9 / 10.9 warp-instructions per clock were such folds)
      if (OP == 4) asm volatile("max.s32 %0, %0, %1;" : "+r"(a[q]) : "r"(b + q));
      if (OP == 5) asm volatile("add.s32 %0, %0, %1;" : "+r"(a[q]) : "r"(b));
      if (OP == 6) a[q] = __viaddmax_s32_relu(a[q], b, c);
      if (OP == 7) a[q] = (int)__viaddmax_s16x2_relu((unsigned)a[q], (unsigned)b, (unsigned)c);
    }
  }
  __syncthreads();
  long long t1 = clock64();
  int s = 0;
  for (int q = 0; q < CH; ++q) s ^= a[q];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

__global__ void __launch_bounds__(1024, 1) k_ffma(const float* in, float* out, long long* cyc) {
  float a[CH], b = in[threadIdx.x & 7], c = in[(threadIdx.x + 3) & 7];
  for (int q = 0; q < CH; ++q) a[q] = in[q] + threadIdx.x;
  __syncthreads();
  long long t0 = clock64();
#pragma unroll 4
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int q = 0; q < CH; ++q) a[q] = fmaf(a[q], b, c);
  }
  __syncthreads();
  long long t1 = clock64();
  float s = 0;
  for (int q = 0; q < CH; ++q) s += a[q];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// LDS.128 bandwidth: each thread streams 16-byte loads from a 64 KB smem buffer.
__global__ void __launch_bounds__(1024, 1) k_lds(const int* in, int* out, long long* cyc) {
  __shared__ int4 buf[2048];
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) buf[i] = make_int4(in[i & 7], i, -i, 1);
  __syncthreads();
  int4 acc = make_int4(0, 0, 0, 0);
  unsigned idx = threadIdx.x;
  long long t0 = clock64();
#pragma unroll 8
  for (int it = 0; it < ITERS; ++it) {
    int4 v = buf[(idx + it * 32) & 2047];
    acc.x ^= v.x; acc.y ^= v.y; acc.z ^= v.z; acc.w ^= v.w;
  }
  __syncthreads();
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc.x ^ acc.y ^ acc.z ^ acc.w;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

__global__ void k_bar(int* out, long long* cyc, int nthreads_unused) {
  int v = threadIdx.x;
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) { __syncthreads(); v += it; }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = v;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

__global__ void k_gridsync(int* out, long long* cyc, int n) {
  cg::grid_group g = cg::this_grid();
  long long t0 = clock64();
  for (int it = 0; it < n; ++it) g.sync();
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  out[blockIdx.x] = n;
}

static double avg(const long long* c, int n) { double s = 0; for (int i = 0; i < n; ++i) s += c[i]; return s / n; }

int main() {
  int dev = 0, nsm = 0, clk = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  CK(cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev));
  int smem_optin = 0, l2 = 0;
  CK(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  CK(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev));
  printf("{\"sms\": %d, \"clock_khz_attr\": %d, \"smem_optin\": %d, \"l2_bytes\": %d}\n", nsm, clk, smem_optin, l2);
  int *din, *dout; float *fin, *fout; long long* dcyc;
  CK(cudaMalloc(&din, 64 * 1024)); CK(cudaMalloc(&dout, nsm * 1024 * 4));
  CK(cudaMalloc(&fin, 64 * 1024)); CK(cudaMalloc(&fout, nsm * 1024 * 4));
  CK(cudaMalloc(&dcyc, nsm * 8 * 64));
  CK(cudaMemset(din, 1, 64 * 1024)); CK(cudaMemset(fin, 0, 64 * 1024));
  long long hc[4096];
  const char* names[8] = {"viaddmax_s32", "viaddmax_s16x2", "vimax3_s32", "vimax3_s16x2_relu",
                          "imax_s32", "iadd_s32", "viaddmax_s32_relu", "viaddmax_s16x2_relu"};
  const int lanes_per_instr[8] = {1, 2, 1, 2, 1, 1, 1, 2};
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  for (int op = 0; op < 8; ++op) {
    for (int rep = 0; rep < 2; ++rep) {
      CK(cudaEventRecord(e0));
      switch (op) {
        case 0: k_alu<0><<<nsm, 1024>>>(din, dout, dcyc); break;
        case 1: k_alu<1><<<nsm, 1024>>>(din, dout, dcyc); break;
        case 2: k_alu<2><<<nsm, 1024>>>(din, dout, dcyc); break;
        case 3: k_alu<3><<<nsm, 1024>>>(din, dout, dcyc); break;
        case 4: k_alu<4><<<nsm, 1024>>>(din, dout, dcyc); break;
        case 5: k_alu<5><<<nsm, 1024>>>(din, dout, dcyc); break;
        case 6: k_alu<6><<<nsm, 1024>>>(din, dout, dcyc); break;
        case 7: k_alu<7><<<nsm, 1024>>>(din, dout, dcyc); break;
      }
      CK(cudaEventRecord(e1)); CK(cudaDeviceSynchronize());
    }
    float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
    CK(cudaMemcpy(hc, dcyc, nsm * 8, cudaMemcpyDeviceToHost));
    double cyc = avg(hc, nsm);
    double instr_per_clk = 1024.0 * ITERS * CH / 32.0 / cyc;  // warp-instructions per SM clock
    double mhz = cyc / (ms * 1e3);
    printf("{\"op\": \"%s\", \"warp_instr_per_clk_sm\": %.3f, \"lane_ops_per_clk_sm\": %.2f, \"eff_mhz\": %.0f, \"ms\": %.4f}\n",
           names[op], instr_per_clk, instr_per_clk * 32 * lanes_per_instr[op], mhz, ms);
  }
  {
    for (int rep = 0; rep < 2; ++rep) { CK(cudaEventRecord(e0)); k_ffma<<<nsm, 1024>>>(fin, fout, dcyc); CK(cudaEventRecord(e1)); CK(cudaDeviceSynchronize()); }
    float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
    CK(cudaMemcpy(hc, dcyc, nsm * 8, cudaMemcpyDeviceToHost));
    double cyc = avg(hc, nsm);
    double ipc = 1024.0 * ITERS * CH / 32.0 / cyc;
    printf("{\"op\": \"ffma\", \"warp_instr_per_clk_sm\": %.3f, \"lane_ops_per_clk_sm\": %.2f, \"eff_mhz\": %.0f}\n", ipc, ipc * 32, cyc / (ms * 1e3));
  }
  {
    CK(cudaFuncSetAttribute(k_lds, cudaFuncAttributeMaxDynamicSharedMemorySize, 0));
    for (int rep = 0; rep < 2; ++rep) { k_lds<<<nsm, 1024>>>(din, dout, dcyc); CK(cudaDeviceSynchronize()); }
    CK(cudaMemcpy(hc, dcyc, nsm * 8, cudaMemcpyDeviceToHost));
    double cyc = avg(hc, nsm);
    printf("{\"op\": \"lds128\", \"bytes_per_clk_sm\": %.2f}\n", 1024.0 * ITERS * 16 / cyc);
  }
  for (int nt : {64, 128, 256, 512, 1024}) {
    for (int rep = 0; rep < 2; ++rep) { k_bar<<<nsm, nt>>>(dout, dcyc, nt); CK(cudaDeviceSynchronize()); }
    CK(cudaMemcpy(hc, dcyc, nsm * 8, cudaMemcpyDeviceToHost));
    printf("{\"op\": \"syncthreads\", \"threads\": %d, \"cycles_per_barrier\": %.1f}\n", nt, avg(hc, nsm) / ITERS);
  }
  for (int bpsm : {1, 2}) {
    int n = 2000;
    int grid = nsm * bpsm;
    void* args[3] = {&dout, &dcyc, &n};
    for (int rep = 0; rep < 2; ++rep) {
      CK(cudaEventRecord(e0));
      CK(cudaLaunchCooperativeKernel((void*)k_gridsync, grid, 256, args, 0, 0));
      CK(cudaEventRecord(e1)); CK(cudaDeviceSynchronize());
    }
    float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
    CK(cudaMemcpy(hc, dcyc, grid * 8, cudaMemcpyDeviceToHost));
    printf("{\"op\": \"grid_sync\", \"ctas\": %d, \"cycles_per_sync\": %.1f, \"us_per_sync\": %.3f}\n", grid, avg(hc, grid) / n, ms * 1e3 / n);
  }
  // launch latency of an empty-ish kernel, back-to-back
  {
    for (int rep = 0; rep < 10; ++rep) k_bar<<<1, 32>>>(dout, dcyc, 0);
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(e0));
    for (int rep = 0; rep < 200; ++rep) k_gridsync<<<1, 32>>>(dout, dcyc, 0);
    CK(cudaEventRecord(e1)); CK(cudaDeviceSynchronize());
    float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
    printf("{\"op\": \"launch_back_to_back\", \"us_per_launch\": %.3f}\n", ms * 1e3 / 200);
  }
  return 0;
}
