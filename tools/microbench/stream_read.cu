// Read-bandwidth microbenchmark for the encode access pattern (SURVEY §7 step 0 style box
// fact): a 4096 x 4096 FP64 matrix (row pitch 32 KiB) read as 128-column chunks of row
// blocks, by (a) plain LDG.64 per thread with many rows in flight, (b) LDG.128, (c) TMA
// bulk copies of one row segment (1 KiB) each into a smem ring, (d) TMA bulk copies of
// 4 KiB segments (512 columns).  Prints one JSON line per variant.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

constexpr int N = 4096;

template <int UNR>
__global__ void __launch_bounds__(128) k_ldg64(const double *__restrict__ A, double *out) {
  const int c = threadIdx.x, chunk = blockIdx.x, I = blockIdx.y;
  const double *src = A + (size_t)I * 64 * N + chunk * 128 + c;
  double s = 0;
  for (int r0 = 0; r0 < 64; r0 += UNR) {
    double v[UNR];
#pragma unroll
    for (int r = 0; r < UNR; ++r) v[r] = __ldg(src + (size_t)(r0 + r) * N);
#pragma unroll
    for (int r = 0; r < UNR; ++r) s += v[r];
  }
  if (s == 12345.0) out[0] = s;
}

template <int UNR>
__global__ void __launch_bounds__(256) k_ldg128(const double *__restrict__ A, double *out) {
  // 64 threads per 128-column row segment, 4 rows per pass
  const int t = threadIdx.x, chunk = blockIdx.x, I = blockIdx.y;
  const int c2 = t & 63, rsub = t >> 6;
  const double2 *src = reinterpret_cast<const double2 *>(A + (size_t)I * 64 * N + chunk * 128) + c2;
  double s = 0;
  for (int r0 = 0; r0 < 64; r0 += 4 * UNR) {
    double2 v[UNR];
#pragma unroll
    for (int r = 0; r < UNR; ++r) v[r] = __ldg(src + (size_t)(r0 + 4 * r + rsub) * (N / 2));
#pragma unroll
    for (int r = 0; r < UNR; ++r) s += v[r].x + v[r].y;
  }
  if (s == 12345.0) out[0] = s;
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t n) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(n)); }
__device__ __forceinline__ void mbar_expect(uint64_t *b, uint32_t bytes) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory"); }
__device__ __forceinline__ void mbar_arrive(uint64_t *b) { asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory"); }
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t ph) {
  asm volatile("{\n.reg .pred P1;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra W_%=;\n}\n" ::"r"(smem_u32(b)), "r"(ph) : "memory");
}
__device__ __forceinline__ void bulk(void *dst, const void *src, uint32_t bytes, uint64_t *b) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(b)) : "memory");
}

// persistent: producer warp streams strips of 16 rows x SEG columns; 4 consumer warps sum
template <int SEG, int STAGES>
__global__ void __launch_bounds__(160) k_bulk(const double *__restrict__ A, double *out, int units) {
  extern __shared__ __align__(16) unsigned char sm[];
  double *ring = reinterpret_cast<double *>(sm);
  __shared__ __align__(8) uint64_t full[STAGES], empty[STAGES];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int u0 = (long)units * blockIdx.x / gridDim.x, u1 = (long)units * (blockIdx.x + 1) / gridDim.x;
  constexpr int NCH = N / SEG;
  if (tid == 0) { for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 4); } asm volatile("fence.mbarrier_init.release.cluster;"); }
  __syncthreads();
  if (warp == 4) {
    if (lane == 0) {
      long it = 0;
      for (int u = u0; u < u1; ++u) {
        const int I = u / NCH, ch = u % NCH;
        for (int s = 0; s < 4; ++s, ++it) {  // 64 rows = 4 strips of 16
          const int st = it % STAGES;
          if (it >= STAGES) mbar_wait(&empty[st], ((it / STAGES) + 1) & 1);
          mbar_expect(&full[st], 16 * SEG * 8);
          for (int r = 0; r < 16; ++r)
            bulk(ring + (size_t)st * 16 * (SEG + 2) + r * (SEG + 2), A + (size_t)(I * 64 + s * 16 + r) * N + ch * SEG, SEG * 8, &full[st]);
        }
      }
    }
    return;
  }
  double acc = 0;
  long it = 0;
  for (int u = u0; u < u1; ++u)
    for (int s = 0; s < 4; ++s, ++it) {
      const int st = it % STAGES;
      mbar_wait(&full[st], (it / STAGES) & 1);
      const double *t = ring + (size_t)st * 16 * (SEG + 2);
      for (int c = tid; c < SEG; c += 128)
        for (int r = 0; r < 16; ++r) acc += t[r * (SEG + 2) + c];
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[st]);
    }
  if (acc == 12345.0) out[0] = acc;
}

__global__ void fill(double *A) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < (size_t)N * N; i += (size_t)gridDim.x * blockDim.x) {
    uint64_t z = i * 0x9E3779B97F4A7C15ull; z ^= z >> 29; z *= 0xBF58476D1CE4E5B9ull; z ^= z >> 32;
    A[i] = (double)(z >> 11) * 0x1.0p-53 * 2.0 - 1.0;
  }
}

template <typename F>
float time_it(F f, int reps = 20) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  for (int i = 0; i < 3; ++i) f();
  cudaEventRecord(a);
  for (int i = 0; i < reps; ++i) f();
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  return ms / reps;
}

template <int SEG, int STAGES>
int run_bulk(const double *A, double *out, int per_sm_req) {
  const size_t smem = (size_t)STAGES * 16 * (SEG + 2) * 8;
  CK(cudaFuncSetAttribute(k_bulk<SEG, STAGES>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int per_sm = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_bulk<SEG, STAGES>, 160, smem));
  if (per_sm_req && per_sm_req < per_sm) per_sm = per_sm_req;
  const int units = (N / 64) * (N / SEG);
  const int grid = 148 * per_sm < units ? 148 * per_sm : units;
  float ms = time_it([&] { k_bulk<SEG, STAGES><<<grid, 160, smem>>>(A, out, units); });
  CK(cudaGetLastError());
  printf("{\"variant\": \"bulk seg=%d stages=%d ctas/sm=%d\", \"us\": %.2f, \"GBps\": %.0f}\n", SEG, STAGES, per_sm, ms * 1e3, (double)N * N * 8 / (ms * 1e6));
  return 0;
}

int main() {
  double *A, *out;
  CK(cudaMalloc(&A, (size_t)N * N * 8));
  CK(cudaMalloc(&out, 64));
  CK(cudaMemset(A, 0, (size_t)N * N * 8));
  if (getenv("RANDOM_FILL")) { fill<<<4096, 256>>>(A); CK(cudaDeviceSynchronize()); printf("{\"fill\": \"random\"}\n"); }
  const double bytes = (double)N * N * 8;
  dim3 g(N / 128, N / 64);
  float ms = time_it([&] { k_ldg64<16><<<g, 128>>>(A, out); });
  printf("{\"variant\": \"ldg64 unroll16\", \"us\": %.2f, \"GBps\": %.0f}\n", ms * 1e3, bytes / (ms * 1e6));
  ms = time_it([&] { k_ldg64<32><<<g, 128>>>(A, out); });
  printf("{\"variant\": \"ldg64 unroll32\", \"us\": %.2f, \"GBps\": %.0f}\n", ms * 1e3, bytes / (ms * 1e6));
  ms = time_it([&] { k_ldg128<8><<<g, 256>>>(A, out); });
  printf("{\"variant\": \"ldg128 unroll8\", \"us\": %.2f, \"GBps\": %.0f}\n", ms * 1e3, bytes / (ms * 1e6));
  ms = time_it([&] { k_ldg128<16><<<g, 256>>>(A, out); });
  printf("{\"variant\": \"ldg128 unroll16\", \"us\": %.2f, \"GBps\": %.0f}\n", ms * 1e3, bytes / (ms * 1e6));
  if (run_bulk<128, 6>(A, out, 0)) return 1;
  if (run_bulk<128, 12>(A, out, 0)) return 1;
  if (run_bulk<128, 6>(A, out, 1)) return 1;
  if (run_bulk<512, 3>(A, out, 0)) return 1;
  if (run_bulk<256, 6>(A, out, 0)) return 1;
  return 0;
}
