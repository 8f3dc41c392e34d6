// cluster_race_probe.cu -- does compute-sanitizer racecheck handle the two DSMEM
// exchange patterns of the cluster kernels, on a minimal kernel?
//   mode 0: every CTA writes a value into its right neighbour's shared memory
//           through a cooperative_groups map_shared_rank pointer, cluster.sync(),
//           reads its own slot (barrier-ordered; no race)
//   mode 1: the same exchange by st.async + mbarrier complete_tx (ordered by the
//           receiver's mbarrier wait)
//   mode 2: mode 0 without the cluster.sync() before the read (a REAL race:
//           racecheck must report it)
//   mode 3: the point-to-point pattern of the cluster kernels: data by st.async
//           on the receiver's mbarrier, and the next round's overwrite of the
//           receiver's slot ordered only by an ACKNOWLEDGEMENT the receiver sends
//           back (st.async on the sender's second mbarrier) after reading --
//           race-free, no cluster barrier inside the loop
// nvcc -gencode arch=compute_100a,code=sm_100a -o tools/cluster_race_probe tools/cluster_race_probe.cu
// compute-sanitizer --tool racecheck tools/cluster_race_probe <mode>
#include <cooperative_groups.h>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
namespace cg = cooperative_groups;

__global__ void __cluster_dims__(4, 1, 1) probe(int mode, int iters, double *out) {
  __shared__ double slot[128];
  __shared__ __align__(8) uint64_t bar, ack;
  __shared__ double token[128];
  cg::cluster_group cl = cg::this_cluster();
  const int rank = cl.block_rank(), t = threadIdx.x;
  const int right = (rank + 1) % 4;
  slot[t] = 0.0;
  if (t == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&ack)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  cl.sync();
  double acc = 0.0;
  uint32_t phase = 0;
  for (int it = 0; it < iters; ++it) {
    const double v = rank * 1000.0 + it + t;
    if (mode == 3) {
      const int left = (rank + 3) % 4;
      auto sa = [](const void *p) { return (uint32_t)__cvta_generic_to_shared(p); };
      uint32_t dslot, dbar, aslot, abar;
      asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(dslot) : "r"(sa(&slot[t])), "r"(right));
      asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(dbar) : "r"(sa(&bar)), "r"(right));
      asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(aslot) : "r"(sa(&token[t])), "r"(left));
      asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(abar) : "r"(sa(&ack)), "r"(left));
      if (it > 0) {  // the right neighbour has read my previous value: its ack arrived
        asm volatile("{\n.reg .pred P;\nA%=:\nmbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P, [%0], %1;\n@!P bra A%=;\n}" ::"r"(
                         sa(&ack)), "r"((phase ^ 1u)) : "memory");
      }
      if (t == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(&bar)), "r"(128 * 8));
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(&ack)), "r"(128 * 8));
      }
      __syncthreads();
      asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b64 [%0], %1, [%2];" ::"r"(dslot),
                   "l"(__double_as_longlong(v)), "r"(dbar) : "memory");
      asm volatile("{\n.reg .pred P;\nW%=:\nmbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P, [%0], %1;\n@!P bra W%=;\n}" ::"r"(
                       sa(&bar)), "r"(phase) : "memory");
      acc += slot[t];
      __syncthreads();  // all of my threads read their slot before the ack leaves
      asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b64 [%0], %1, [%2];" ::"r"(aslot),
                   "l"(__double_as_longlong(acc)), "r"(abar) : "memory");
      phase ^= 1u;
      if (it + 1 == iters)  // drain the last ack before leaving
        asm volatile("{\n.reg .pred P;\nD%=:\nmbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P, [%0], %1;\n@!P bra D%=;\n}" ::"r"(
                         sa(&ack)), "r"((phase ^ 1u)) : "memory");
    } else if (mode == 1) {
      if (t == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(
            (uint32_t)__cvta_generic_to_shared(&bar)), "r"(128 * 8));
      uint32_t raddr, rbar;
      asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(raddr)
                   : "r"((uint32_t)__cvta_generic_to_shared(&slot[t])), "r"(right));
      asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(rbar)
                   : "r"((uint32_t)__cvta_generic_to_shared(&bar)), "r"(right));
      asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b64 [%0], %1, [%2];" ::"r"(raddr),
                   "l"(__double_as_longlong(v)), "r"(rbar) : "memory");
      asm volatile("{\n.reg .pred P;\nW%=:\nmbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P, [%0], %1;\n@!P bra W%=;\n}" ::"r"(
                       (uint32_t)__cvta_generic_to_shared(&bar)), "r"(phase) : "memory");
      phase ^= 1u;
      acc += slot[t];
      cl.sync();  // the next round's writes after everyone read
    } else {
      cl.map_shared_rank(slot, right)[t] = v;
      if (mode == 0) cl.sync();
      acc += slot[t];
      cl.sync();
    }
  }
  cl.sync();
  out[blockIdx.x * 128 + t] = acc;
}

int main(int argc, char **argv) {
  const int mode = argc > 1 ? atoi(argv[1]) : 0;
  double *out;
  cudaMalloc(&out, 8 * 128 * 8);
  probe<<<8, 128>>>(mode, 16, out);
  cudaError_t e = cudaDeviceSynchronize();
  printf("mode %d: %s\n", mode, cudaGetErrorString(e));
  return e != cudaSuccess;
}
