// Step-0 box facts: FP64 DMMA (mma.sync .f64) vs DFMA vs FFMA
// issue throughput on sm_100a, plus an HBM copy. Standalone; prints JSON lines.
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("err %s line %d\n",cudaGetErrorString(e),__LINE__);return 1;}}while(0)

template<int NACC>
__global__ void k_m8n8k4(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
  double c[NACC][2];
  #pragma unroll
  for (int i = 0; i < NACC; ++i) { c[i][0] = 0; c[i][1] = 0; }
  for (int it = 0; it < iters; ++it) {
    #pragma unroll
    for (int i = 0; i < NACC; ++i)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
  }
  double s = 0;
  #pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i][0] + c[i][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template<int NACC>
__global__ void k_m16n8k4(double* out, int iters) {
  double a0 = threadIdx.x * 1e-3, a1 = a0 + 1, b = 1.0 + threadIdx.x * 1e-4;
  double c[NACC][4];
  #pragma unroll
  for (int i = 0; i < NACC; ++i) { c[i][0] = c[i][1] = c[i][2] = c[i][3] = 0; }
  for (int it = 0; it < iters; ++it) {
    #pragma unroll
    for (int i = 0; i < NACC; ++i)
      asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
                   : "+d"(c[i][0]), "+d"(c[i][1]), "+d"(c[i][2]), "+d"(c[i][3]) : "d"(a0), "d"(a1), "d"(b));
  }
  double s = 0;
  #pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i][0] + c[i][1] + c[i][2] + c[i][3];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template<int NACC>
__global__ void k_m16n8k16(double* out, int iters) {
  double a[8], b[4];
  #pragma unroll
  for (int i = 0; i < 8; ++i) a[i] = threadIdx.x * 1e-3 + i;
  #pragma unroll
  for (int i = 0; i < 4; ++i) b[i] = 1.0 + threadIdx.x * 1e-4 + i;
  double c[NACC][4];
  #pragma unroll
  for (int i = 0; i < NACC; ++i) { c[i][0] = c[i][1] = c[i][2] = c[i][3] = 0; }
  for (int it = 0; it < iters; ++it) {
    #pragma unroll
    for (int i = 0; i < NACC; ++i)
      asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};"
                   : "+d"(c[i][0]), "+d"(c[i][1]), "+d"(c[i][2]), "+d"(c[i][3])
                   : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]),
                     "d"(b[0]), "d"(b[1]), "d"(b[2]), "d"(b[3]));
  }
  double s = 0;
  #pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i][0] + c[i][1] + c[i][2] + c[i][3];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template<int NACC>
__global__ void k_dfma(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-9;
  double c[NACC];
  #pragma unroll
  for (int i = 0; i < NACC; ++i) c[i] = i;
  for (int it = 0; it < iters; ++it) {
    #pragma unroll
    for (int i = 0; i < NACC; ++i) c[i] = fma(c[i], b, a);
  }
  double s = 0;
  #pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template<int NACC>
__global__ void k_ffma(float* out, int iters) {
  float a = threadIdx.x * 1e-3f, b = 1.0f + threadIdx.x * 1e-7f;
  float c[NACC];
  #pragma unroll
  for (int i = 0; i < NACC; ++i) c[i] = i;
  for (int it = 0; it < iters; ++it) {
    #pragma unroll
    for (int i = 0; i < NACC; ++i) c[i] = fmaf(c[i], b, a);
  }
  float s = 0;
  #pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// packed fp32x2 FMA (sm_100 FFMA2) with a broadcast scalar operand -- the FP32 GEMM's form
template<int NACC>
__global__ void k_ffma2(float* out, int iters) {
  const float a = threadIdx.x * 1e-3f;
  const float2 b = make_float2(1.0f + threadIdx.x * 1e-7f, 1.0f - threadIdx.x * 1e-7f);
  float2 c[NACC];
  #pragma unroll
  for (int i = 0; i < NACC; ++i) c[i] = make_float2(i, -i);
  for (int it = 0; it < iters; ++it) {
    #pragma unroll
    for (int i = 0; i < NACC; ++i) c[i] = __ffma2_rn(make_float2(a, a), b, c[i]);
  }
  float s = 0;
  #pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i].x + c[i].y;
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void k_copy(const double4* __restrict__ a, double4* __restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}

// best of `reps` timed launches; a launch that fails (e.g. too many registers for the block
// size) returns -1 so no rate is printed for it (r01's impossible rows came from timing a
// failed launch)
template<class F>
float time_it(F f, int reps) {
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  f();
  if (cudaGetLastError() != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) return -1.f;
  float best = 1e30f;
  for (int r = 0; r < reps; ++r) {
    cudaEventRecord(e0); f(); cudaEventRecord(e1);
    if (cudaGetLastError() != cudaSuccess || cudaEventSynchronize(e1) != cudaSuccess) return -1.f;
    float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
  }
  return best;
}

void report(const char *kernel, int wpb, double flop, float ms) {
  if (ms <= 0.f) printf("{\"kernel\":\"%s\",\"warps_per_block\":%d,\"tflops\":null,\"error\":\"launch failed\"}\n", kernel, wpb);
  else printf("{\"kernel\":\"%s\",\"warps_per_block\":%d,\"tflops\":%.3f}\n", kernel, wpb, flop / (ms * 1e9));
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* out; CK(cudaMalloc(&out, 1 << 26));
  const int iters = 4096;
  for (int wpb : {4, 8, 16, 32}) {
    int threads = wpb * 32, blocks = sms * 2;
    size_t warps = (size_t)blocks * wpb;
    float ms;
    ms = time_it([&] { k_m8n8k4<8><<<blocks, threads>>>(out, iters); }, 5);
    report("dmma_m8n8k4", wpb, warps * iters * 8.0 * 512, ms);
    ms = time_it([&] { k_m16n8k4<8><<<blocks, threads>>>(out, iters); }, 5);
    report("dmma_m16n8k4", wpb, warps * iters * 8.0 * 1024, ms);
    ms = time_it([&] { k_m16n8k16<8><<<blocks, threads>>>(out, iters / 4); }, 5);
    report("dmma_m16n8k16", wpb, warps * (iters / 4) * 8.0 * 4096, ms);
    ms = time_it([&] { k_dfma<16><<<blocks, threads>>>(out, iters); }, 5);
    report("dfma", wpb, warps * 32.0 * iters * 16 * 2, ms);
    ms = time_it([&] { k_ffma<16><<<blocks, threads>>>((float*)out, iters); }, 5);
    report("ffma", wpb, warps * 32.0 * iters * 16 * 2, ms);
    ms = time_it([&] { k_ffma2<16><<<blocks, threads>>>((float*)out, iters); }, 5);
    report("ffma2", wpb, warps * 32.0 * iters * 16 * 4, ms);
  }
  size_t bytes = (size_t)2 << 30; double4 *a, *b;
  CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes)); cudaMemset(a, 0, bytes);
  float ms = time_it([&] { k_copy<<<sms * 8, 256>>>(a, b, bytes / 32); }, 10);
  printf("{\"kernel\":\"hbm_copy\",\"gbs\":%.1f}\n", 2.0 * bytes / (ms * 1e6));
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("{\"sms\":%d,\"clock_khz\":%d}\n", sms, clk);
  return 0;
}
