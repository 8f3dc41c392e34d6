// tmem_probe.cu -- measure tcgen05.ld (TMEM -> registers) throughput per SM.
// Question: can TMEM hold matrix values next to SMEM (a separate read path)?
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/tmem_probe tools/tmem_probe.cu
// Each CTA (NT threads = NT/32 warps, warp w reads TMEM lanes 32*(w%4)..+31)
// allocates COLS columns, fills them with tcgen05.st, then loops tcgen05.ld
// of X columns (x X 32-bit registers per thread) + wait::ld, summing.
#include <cstdio>
#include <cstdint>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

template <int X>
__device__ __forceinline__ void tmem_ld(uint32_t taddr, uint32_t (&r)[X]);

template <>
__device__ __forceinline__ void tmem_ld<16>(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
}

__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
      "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]));
}

template <int NT, int COLS>
__global__ void __launch_bounds__(NT) probe(int iters, int lds_per_wait, double *sink, long long *cyc) {
  __shared__ uint32_t taddr_s;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     (uint32_t)__cvta_generic_to_shared(&taddr_s)),
                 "n"(COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t base = taddr_s + ((uint32_t)(32 * (warp & 3)) << 16);
  // warps >= 4 share lane quarters with warps w-4: give them another column half
  const uint32_t colbase = (warp >> 2) * (COLS / 2);
  uint32_t v[16];
  for (int i = 0; i < 16; ++i) v[i] = threadIdx.x * 16 + i;
  for (int c = 0; c < COLS / 2; c += 16) tmem_st16(base + colbase + c, v);
  asm volatile("tcgen05.wait::st.sync.aligned;");
  __syncthreads();
  uint32_t acc = 0;
  const long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
    if (lds_per_wait == 4) {
      uint32_t r0[16], r1[16], r2[16], r3[16];
      const uint32_t c = base + colbase + ((it * 64) % (COLS / 2));
      tmem_ld<16>(c, r0);
      tmem_ld<16>(c + 16, r1);
      tmem_ld<16>(c + 32, r2);
      tmem_ld<16>(c + 48, r3);
      asm volatile("tcgen05.wait::ld.sync.aligned;");
#pragma unroll
      for (int i = 0; i < 16; ++i) acc += r0[i] ^ r1[i] ^ r2[i] ^ r3[i];
    } else {
      uint32_t r[16];
      tmem_ld<16>(base + colbase + ((it * 16) % (COLS / 2)), r);
      asm volatile("tcgen05.wait::ld.sync.aligned;");
#pragma unroll
      for (int i = 0; i < 16; ++i) acc += r[i];
    }
  }
  const long long c1 = clock64();
  if (acc == 0xdeadbeef) sink[blockIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr_s), "n"(COLS));
}

template <int NT, int COLS>
int run(int ctas_per_sm, int iters, int lpw = 1) {
  int dev = 0, sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int grid = sms * ctas_per_sm;
  double *sink;
  long long *cyc;
  CK(cudaMalloc(&sink, grid * 8));
  CK(cudaMalloc(&cyc, grid * 8));
  probe<NT, COLS><<<grid, NT>>>(16, 1, sink, cyc);
  CK(cudaDeviceSynchronize());
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  probe<NT, COLS><<<grid, NT>>>(iters, lpw, sink, cyc);
  cudaEventRecord(b);
  CK(cudaEventSynchronize(b));
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  std::vector<long long> hc(grid);
  cudaMemcpy(hc.data(), cyc, grid * 8, cudaMemcpyDeviceToHost);
  long long mx = 0;
  for (auto c : hc) mx = c > mx ? c : mx;
  const double bytes = (double)grid * NT * iters * 16 * 4 * lpw;
  printf("NT=%d COLS=%d ctas/SM=%d loads/wait=%d: %.1f TB/s total, %.1f B/clk/SM (clk %.0f MHz)\n",
         NT, COLS, ctas_per_sm, lpw, bytes / (ms * 1e-3) / 1e12, bytes / sms / (double)mx,
         mx / (ms * 1e3));
  cudaFree(sink);
  cudaFree(cyc);
  return 0;
}

int main() {
  run<128, 256>(1, 1 << 13, 4);
  run<128, 256>(2, 1 << 13, 4);
  run<256, 256>(1, 1 << 13, 4);
  run<256, 256>(2, 1 << 13, 4);
  run<512, 256>(1, 1 << 13, 4);
  run<512, 256>(1, 1 << 13, 1);
  return 0;
}
