// TMEM load / store throughput probe (sm_100a): cycles per tcgen05.ld/st of 32 lanes x 32 columns.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tmem_probe tmem_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int MODE, int INFL>
__global__ void k_probe(int iters, unsigned long long* out, uint32_t* sink) {
  __shared__ uint32_t tbase;
  const int wid = threadIdx.x >> 5;
  if (wid == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_addr(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = tbase + ((uint32_t)(32 * (wid & 3)) << 16);
  const int nw = blockDim.x >> 5;
  uint32_t acc = 0;
  uint32_t v[INFL][32];
  for (int k = 0; k < INFL; ++k)
    for (int j = 0; j < 32; ++j) v[k][j] = j + threadIdx.x;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int k = 0; k < INFL; ++k) {
      const uint32_t col = (uint32_t)(((it * INFL + k) * 32 + (wid >> 2) * 128) & 511);
      if (MODE == 0) {
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
            "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
            : "=r"(v[k][0]), "=r"(v[k][1]), "=r"(v[k][2]), "=r"(v[k][3]), "=r"(v[k][4]), "=r"(v[k][5]), "=r"(v[k][6]),
              "=r"(v[k][7]), "=r"(v[k][8]), "=r"(v[k][9]), "=r"(v[k][10]), "=r"(v[k][11]), "=r"(v[k][12]),
              "=r"(v[k][13]), "=r"(v[k][14]), "=r"(v[k][15]), "=r"(v[k][16]), "=r"(v[k][17]), "=r"(v[k][18]),
              "=r"(v[k][19]), "=r"(v[k][20]), "=r"(v[k][21]), "=r"(v[k][22]), "=r"(v[k][23]), "=r"(v[k][24]),
              "=r"(v[k][25]), "=r"(v[k][26]), "=r"(v[k][27]), "=r"(v[k][28]), "=r"(v[k][29]), "=r"(v[k][30]),
              "=r"(v[k][31])
            : "r"(tb + col));
      } else {
        asm volatile(
            "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
            "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(tb + col),
            "r"(v[k][0]), "r"(v[k][1]), "r"(v[k][2]), "r"(v[k][3]), "r"(v[k][4]), "r"(v[k][5]), "r"(v[k][6]),
            "r"(v[k][7]), "r"(v[k][8]), "r"(v[k][9]), "r"(v[k][10]), "r"(v[k][11]), "r"(v[k][12]), "r"(v[k][13]),
            "r"(v[k][14]), "r"(v[k][15]), "r"(v[k][16]), "r"(v[k][17]), "r"(v[k][18]), "r"(v[k][19]),
            "r"(v[k][20]), "r"(v[k][21]), "r"(v[k][22]), "r"(v[k][23]), "r"(v[k][24]), "r"(v[k][25]),
            "r"(v[k][26]), "r"(v[k][27]), "r"(v[k][28]), "r"(v[k][29]), "r"(v[k][30]), "r"(v[k][31])
            : "memory");
      }
    }
    if (MODE == 0) {
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
      for (int k = 0; k < INFL; ++k)
#pragma unroll
        for (int j = 0; j < 32; ++j) acc ^= v[k][j];
    } else {
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
#pragma unroll
      for (int k = 0; k < INFL; ++k) v[k][it & 31] += 1;
    }
  }
  long long t1 = clock64();
  __syncthreads();
  if (threadIdx.x == 0) atomicAdd(out, (unsigned long long)(t1 - t0));
  if (acc == 0x12345) sink[0] = acc;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (wid == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
}

template <int MODE, int INFL>
void run(int warps) {
  unsigned long long* d;
  uint32_t* s;
  cudaMalloc(&d, 8);
  cudaMalloc(&s, 8);
  cudaMemset(d, 0, 8);
  const int iters = 2000;
  k_probe<MODE, INFL><<<148, 32 * warps>>>(iters, d, s);
  cudaMemset(d, 0, 8);
  k_probe<MODE, INFL><<<148, 32 * warps>>>(iters, d, s);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned long long h = 0;
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  const double cyc = (double)h / 148.0;  // per CTA (= per SM)
  const double bytes = (double)iters * INFL * warps * 32 * 32 * 4;
  printf("%s x32 warps=%2d inflight=%d: %.1f B/clk/SM (%.1f clk per warp-instr) %s\n", MODE ? "st" : "ld", warps, INFL,
         bytes / cyc, cyc / ((double)iters * INFL), cudaGetErrorString(e));
  cudaFree(d);
  cudaFree(s);
}

int main() {
  run<0, 1>(4);
  run<0, 2>(4);
  run<0, 1>(8);
  run<0, 2>(8);
  run<0, 1>(16);
  run<0, 2>(16);
  run<1, 1>(4);
  run<1, 1>(8);
  run<1, 2>(8);
  return 0;
}
