// Encode-kernel harness: the library's encode_a/encode_b kernels (compiled in from
// csrc/encode.cu) timed cold-ish against a plain streaming read of the same matrix.
#include <cstdarg>
#include <cstdio>
#include "../../paper_conf_dsn_braunhw14_b200/csrc/encode.cu"
namespace aabft {
void set_error(const char *, ...) {}
int64_t next_launch(int64_t n) { return n; }
aabft_status check_launch(const char *w) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) { printf("cuda error %s: %s\n", w, cudaGetErrorString(e)); return AABFT_ECUDA; }
  return AABFT_OK;
}
}  // namespace aabft
using namespace aabft;
int main(int argc, char **argv) {
  const int n = 4096, bs = 64, P = 2;
  double *A, *Acs, *Bcs, *tav, *tbv, *flush;
  int *tai, *tbi;
  cudaMalloc(&A, (size_t)n * n * 8);
  cudaMalloc(&flush, (size_t)256 << 20);
  cudaMalloc(&Acs, (size_t)n / bs * n * 8);
  cudaMalloc(&Bcs, (size_t)n * (n / bs) * 8);
  cudaMalloc(&tav, (size_t)(n + n / bs) * P * 8);
  cudaMalloc(&tbv, (size_t)(n + n / bs) * P * 8);
  cudaMalloc(&tai, (size_t)(n + n / bs) * P * 4);
  cudaMalloc(&tbi, (size_t)(n + n / bs) * P * 4);
  cudaMemset(A, 0, (size_t)n * n * 8);
  aabft_config cfg{};
  cfg.dtype = AABFT_F64; cfg.M = cfg.N = cfg.K = n; cfg.bs = bs; cfg.p = P; cfg.omega = 3; cfg.fma_model = 1;
  void *ws;
  cudaMalloc(&ws, encode_ws_bytes(&cfg) + 256);
  aabft_encoded enc{Acs, n, Bcs, n / bs, tav, tai, tbv, tbi};
  aabft_encoded enc_cs{Acs, n, Bcs, n / bs, nullptr, nullptr, nullptr, nullptr};
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  auto timeit = [&](const char *name, auto fn) {
    float tot = 0; int reps = 10;
    for (int r = 0; r < reps + 2; ++r) {
      cudaMemsetAsync(flush, r, (size_t)256 << 20);  // evict L2
      cudaEventRecord(e0);
      fn();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      if (r >= 2) tot += ms;
    }
    printf("{\"kernel\": \"%s\", \"us\": %.2f, \"GBps\": %.0f}\n", name, tot / reps * 1e3, (double)n * n * 8 / (tot / reps * 1e6));
  };
  timeit("encode A (top-p)", [&] { launch_encode(&cfg, A, n, nullptr, 0, &enc, ws, 0); });
  timeit("encode A (checksums only)", [&] { launch_encode(&cfg, A, n, nullptr, 0, &enc_cs, ws, 0); });
  timeit("encode B (top-p)", [&] { launch_encode(&cfg, nullptr, 0, A, n, &enc, ws, 0); });
  timeit("encode B (checksums only)", [&] { launch_encode(&cfg, nullptr, 0, A, n, &enc_cs, ws, 0); });
  cudaDeviceSynchronize();
  printf("{\"status\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
