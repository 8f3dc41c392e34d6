// dsmem_probe.cu -- round-trip latency of the cluster exchange primitives on
// B200 (sm_100a), to decide how the n = 4032 cluster plan (line3_kernel.cuh)
// should move its reduction partials and halo rows.  A cluster of 2 CTAs
// ping-pongs N times; one elected thread per CTA (or a whole warp for the
// per-element variants) sends, the peer waits on its mbarrier, then answers.
//   mode 0: st.async 8 B (mbarrier complete_tx) -- the reduction partials
//   mode 1: cp.async.bulk smem -> peer smem, 80 B (complete_tx)
//   mode 2: cp.async.bulk 1040 B (one halo-state side of 2 fields)
//   mode 3: st.shared::cluster 8 B + mbarrier.arrive.release.cluster (remote)
//   mode 4: 32 lanes x st.async 8 B (a warp-wide element push)
//   mode 5: mode 1 preceded by fence.proxy.async.shared::cta
// Prints cycles per one-way hop (round trip / 2).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/dsmem_probe tools/dsmem_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t r) {
  uint32_t o;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(o) : "r"(a), "r"(r));
  return o;
}
__device__ __forceinline__ void wait_parity(uint32_t bar, uint32_t ph) {
  asm volatile(
      "{\n\t.reg .pred P;\nW_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra W_%=;\n}" ::"r"(bar),
      "r"(ph)
      : "memory");
}

template <int MODE>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(32) probe(int iters, long long *out) {
  __shared__ __align__(16) double buf[256];
  __shared__ __align__(16) double src[256];
  __shared__ __align__(8) uint64_t bar;
  uint32_t rank;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  const int l = threadIdx.x;
  for (int i = l; i < 256; i += 32) src[i] = i;
  const uint32_t cnt = MODE == 3 ? 1u : 1u;
  if (l == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(&bar)), "r"(cnt));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  const uint32_t peer = rank ^ 1u;
  const uint32_t rbuf = mapa(sa(buf), peer), rbar = mapa(sa(&bar), peer);
  const uint32_t mybar = sa(&bar);
  const uint32_t bytes = MODE == 0 ? 8u : MODE == 1 || MODE == 5 ? 80u : MODE == 2 ? 1040u
                         : MODE == 4 ? 256u : 0u;
  uint32_t ph = 0;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    const bool my_turn = ((it & 1) == 0) == (rank == 0);
    // arm my barrier for the message I will receive this round (receiver side)
    if (!my_turn) {
      if (l == 0) {
        if (MODE == 3)
          ;  // arrival comes from the peer's remote arrive
        else
          asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mybar), "r"(bytes)
                       : "memory");
      }
      wait_parity(mybar, ph);
      ph ^= 1u;
      __syncwarp();
    } else {
      if (MODE == 0 && l == 0) {
        asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b64 [%0], %1, [%2];" ::"r"(rbuf),
                     "l"((long long)it), "r"(rbar)
                     : "memory");
      } else if ((MODE == 1 || MODE == 2 || MODE == 5) && l == 0) {
        if (MODE == 5) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile(
            "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                rbuf),
            "r"(sa(src)), "r"(bytes), "r"(rbar)
            : "memory");
      } else if (MODE == 3 && l == 0) {
        asm volatile("st.shared::cluster.f64 [%0], %1;" ::"r"(rbuf), "d"((double)it) : "memory");
        asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(rbar) : "memory");
      } else if (MODE == 4) {
        asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b64 [%0], %1, [%2];" ::"r"(
                         rbuf + 8u * l),
                     "l"((long long)it), "r"(rbar)
                     : "memory");
      }
      __syncwarp();
    }
  }
  long long t1 = clock64();
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (l == 0 && rank == 0) out[blockIdx.x / 2] = (t1 - t0);
}

template <int MODE>
void run(const char *name) {
  long long *d, h[1];
  cudaMalloc(&d, sizeof(long long));
  const int iters = 20000;
  probe<MODE><<<2, 32>>>(100, d);
  cudaDeviceSynchronize();
  probe<MODE><<<2, 32>>>(iters, d);
  cudaError_t e = cudaDeviceSynchronize();
  cudaMemcpy(h, d, sizeof(long long), cudaMemcpyDeviceToHost);
  printf("mode %d %-44s %s  %.1f cycles per one-way hop\n", MODE, name, cudaGetErrorString(e),
         (double)h[0] / iters);
  cudaFree(d);
}

int main() {
  run<0>("st.async 8 B + complete_tx");
  run<1>("cp.async.bulk 80 B smem->peer");
  run<2>("cp.async.bulk 1040 B smem->peer");
  run<3>("st.shared::cluster + remote arrive.release");
  run<4>("32 lanes x st.async 8 B");
  run<5>("fence.proxy.async + cp.async.bulk 80 B");
  return 0;
}
