// pdl_probe.cu -- can a small one-CTA-per-SM grid share the GPU with a 3-CTA-per-SM persistent
// grid launched after it as a programmatic dependent launch?  Mimics the resource footprint of
// encode_overlap_kernel (64 threads, 64 registers, ~21 KB smem) and gemm_f64_kernel (160
// threads, 128 registers, 68.7 KB smem, 444 CTAs).  Prints when the secondary CTAs start
// relative to the primary's start / end, per SM residency.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o pdl_probe pdl_probe.cu && ./pdl_probe
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned smid() {
  unsigned s;
  asm volatile("mov.u32 %0, %smid;" : "=r"(s));
  return s;
}

__global__ void __launch_bounds__(64, 16) prim(unsigned long long *rec, long long spin_ns) {
  extern __shared__ unsigned char sm[];
#ifndef NO_TRIGGER
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
  const unsigned long long t0 = gtime();
  if (threadIdx.x == 0) { sm[0] = 1; rec[blockIdx.x * 3] = t0; rec[blockIdx.x * 3 + 1] = smid(); }
  while (gtime() - t0 < (unsigned long long)spin_ns) {}
  if (threadIdx.x == 0) rec[blockIdx.x * 3 + 2] = gtime();
}

__global__ void __launch_bounds__(160, 3) sec(unsigned long long *rec, long long work_ns) {
  extern __shared__ unsigned char sm[];
  const unsigned long long t0 = gtime();
  if (threadIdx.x == 0) { sm[0] = 1; rec[blockIdx.x * 3] = t0; rec[blockIdx.x * 3 + 1] = smid(); }
  while (gtime() - t0 < (unsigned long long)work_ns) {}
  if (threadIdx.x == 0) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    rec[blockIdx.x * 3 + 2] = gtime();
  }
}

int main(int argc, char **argv) {
  const int prim_smem = argc > 1 ? atoi(argv[1]) : 20640;
  const int sec_smem = argc > 2 ? atoi(argv[2]) : 68736;
  const int nprim = argc > 3 ? atoi(argv[3]) : 128;
  const int nsec = argc > 4 ? atoi(argv[4]) : 444;
  int v = 0;
  cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerMultiprocessor, 0);
  int r = 0;
  cudaDeviceGetAttribute(&r, cudaDevAttrReservedSharedMemoryPerBlock, 0);
  printf("smem per SM %d, reserved per block %d\n", v, r);
  cudaFuncSetAttribute(prim, cudaFuncAttributeMaxDynamicSharedMemorySize, prim_smem);
  cudaFuncSetAttribute(sec, cudaFuncAttributeMaxDynamicSharedMemorySize, sec_smem);
  cudaFuncSetAttribute(prim, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  cudaFuncSetAttribute(sec, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, sec, 160, sec_smem);
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, prim);
  printf("prim regs %d, sec occupancy %d\n", fa.numRegs, occ);
  cudaFuncGetAttributes(&fa, sec);
  printf("sec regs %d\n", fa.numRegs);
  unsigned long long *rp, *rs;
  cudaMalloc(&rp, nprim * 3 * 8);
  cudaMalloc(&rs, nsec * 3 * 8);
  for (int it = 0; it < 3; ++it) {
    prim<<<nprim, 64, prim_smem>>>(rp, 500000);
    cudaLaunchConfig_t lc = {};
    lc.gridDim = dim3(nsec);
    lc.blockDim = dim3(160);
    lc.dynamicSmemBytes = sec_smem;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    lc.attrs = at;
    lc.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&lc, sec, rs, (long long)200000);
    if (e != cudaSuccess) { printf("launch: %s\n", cudaGetErrorString(e)); return 1; }
    e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("sync: %s\n", cudaGetErrorString(e)); return 1; }
  }
  std::vector<unsigned long long> hp(nprim * 3), hs(nsec * 3);
  cudaMemcpy(hp.data(), rp, hp.size() * 8, cudaMemcpyDeviceToHost);
  cudaMemcpy(hs.data(), rs, hs.size() * 8, cudaMemcpyDeviceToHost);
  unsigned long long p0 = ~0ull, p1 = 0;
  std::vector<int> per_sm(200, 0);
  for (int i = 0; i < nprim; ++i) { p0 = std::min(p0, hp[i * 3]); p1 = std::max(p1, hp[i * 3 + 2]); per_sm[hp[i * 3 + 1]]++; }
  int maxp = *std::max_element(per_sm.begin(), per_sm.end());
  std::vector<double> st;
  for (int i = 0; i < nsec; ++i) st.push_back((double)(hs[i * 3] - p0) / 1000.0);
  std::sort(st.begin(), st.end());
  int early = 0;
  for (double s : st) early += s < (p1 - p0) / 1000.0;
  printf("primary: %.1f us, max CTAs per SM %d\n", (p1 - p0) / 1000.0, maxp);
  printf("secondary start (us after primary start): min %.1f p50 %.1f p90 %.1f max %.1f; %d of %d started before the primary ended\n",
         st.front(), st[st.size() / 2], st[st.size() * 9 / 10], st.back(), early, nsec);
  return 0;
}
