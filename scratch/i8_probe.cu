// Probe: tcgen05.mma kind::i8, A (int8, 128 x 128) in TMEM, B (int8, N x 128) in shared memory
// (MN-major or K-major, no swizzle), D int32 in TMEM.  Compares with a CPU product.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o i8_probe i8_probe.cu
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;
  return d;
}
constexpr int N = 64, K = 128, M = 128;

__global__ void k_probe(const int8_t* A, const int8_t* B, int32_t* D, int mode, int lbo, int sbo) {
  __shared__ __align__(1024) int8_t bs[N * K];
  __shared__ uint32_t tbase;
  __shared__ __align__(8) uint64_t bar;
  const int tid = threadIdx.x, wid = tid >> 5;
  // B into shared memory
  for (int t = tid; t < N * K; t += blockDim.x) {
    const int n = t / K, k = t % K;
    int off;
    if (mode == 0)  // MN-major: (n/16)*SBO + (k/8)*LBO + (k%8)*16 + (n%16)
      off = (n / 16) * sbo + (k / 8) * lbo + (k % 8) * 16 + (n % 16);
    else  // K-major: (n/8)*SBO + (k/16)*LBO + (n%8)*16 + (k%16)
      off = (n / 8) * sbo + (k / 16) * lbo + (n % 8) * 16 + (k % 16);
    bs[off] = B[n * K + k];
  }
  if (wid == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_addr(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = tbase;
  // A row `tid` into TMEM columns [0, 32): word w = bytes A[row][4w..4w+3]
  {
    uint32_t v[32];
    for (int w = 0; w < 32; ++w) {
      uint32_t x = 0;
      for (int b = 0; b < 4; ++b) x |= (uint32_t)(uint8_t)A[tid * K + 4 * w + b] << (8 * b);
      v[w] = x;
    }
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
        "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(tb + ((uint32_t)(32 * wid) << 16)),
        "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]), "r"(v[9]),
        "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15]), "r"(v[16]), "r"(v[17]), "r"(v[18]),
        "r"(v[19]), "r"(v[20]), "r"(v[21]), "r"(v[22]), "r"(v[23]), "r"(v[24]), "r"(v[25]), "r"(v[26]), "r"(v[27]),
        "r"(v[28]), "r"(v[29]), "r"(v[30]), "r"(v[31])
        : "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  if (tid == 0) {
    // idesc: D s32 (2<<4), A s8 (1<<7), B s8 (1<<10), B major (mode 0: MN -> 1), N>>3 << 17, M>>4 << 24
    const uint32_t idesc = (2u << 4) | (1u << 7) | (1u << 10) | ((mode == 0 ? 1u : 0u) << 16) | ((uint32_t)(N >> 3) << 17) |
                           ((uint32_t)(M >> 4) << 24);
    const uint32_t bsa = smem_addr(bs);
    for (int kk = 0; kk < K / 32; ++kk) {
      // 32 K-values: MN-major -> 4 core-matrix rows of 8 along K (4 * LBO); K-major -> 2 * LBO
      const uint32_t boff = mode == 0 ? kk * 4 * lbo : kk * 2 * lbo;
      const uint64_t bd = mode == 0 ? sdesc(bsa + boff, lbo, sbo) : sdesc(bsa + boff, lbo, sbo);
      const uint32_t acc = kk > 0;
      asm volatile(
          "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
          " tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n}" ::"r"(tb + 64),
          "r"(tb + 8 * kk), "l"(bd), "r"(idesc), "r"(acc)
          : "memory");
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_addr(&bar))
                 : "memory");
  }
  __syncwarp();
  asm volatile(
      "{\n .reg .pred p;\n WAIT:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra WAIT;\n}" ::"r"(
          smem_addr(&bar))
      : "memory");
  asm volatile("tcgen05.fence::after_thread_sync;");
  for (int c = 0; c < N; c += 8) {
    uint32_t v[8];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "r"(tb + ((uint32_t)(32 * wid) << 16) + 64 + c));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    for (int j = 0; j < 8; ++j) D[tid * N + c + j] = (int32_t)v[j];
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (wid == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tb));
}

int main() {
  int8_t hA[M * K], hB[N * K];
  srand(1);
  for (int i = 0; i < M * K; ++i) hA[i] = (rand() % 3 == 0) ? -1 : ((rand() % 7 == 0) ? (int8_t)(rand() % 256 - 128) : 0);
  for (int i = 0; i < N * K; ++i) hB[i] = (int8_t)(rand() % 256 - 128);
  int ref[M * N];
  for (int m = 0; m < M; ++m)
    for (int n = 0; n < N; ++n) {
      int s = 0;
      for (int k = 0; k < K; ++k) s += hA[m * K + k] * hB[n * K + k];
      ref[m * N + n] = s;
    }
  int8_t *dA, *dB;
  int32_t* dD;
  cudaMalloc(&dA, sizeof hA);
  cudaMalloc(&dB, sizeof hB);
  cudaMalloc(&dD, M * N * 4);
  cudaMemcpy(dA, hA, sizeof hA, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB, sizeof hB, cudaMemcpyHostToDevice);
  struct Cfg { int mode, lbo, sbo; const char* name; } cfgs[] = {
      {0, 128, 2048, "MN-major LBO=128(K) SBO=2048(MN)"},
      {0, 2048, 128, "MN-major LBO=2048 SBO=128 (swapped)"},
      {1, 128, 1024, "K-major LBO=128(K) SBO=1024(N)"},
      {1, 1024, 128, "K-major LBO=1024 SBO=128 (swapped)"},
  };
  for (auto& c : cfgs) {
    cudaMemset(dD, 0, M * N * 4);
    k_probe<<<1, 128>>>(dA, dB, dD, c.mode, c.lbo, c.sbo);
    cudaError_t e = cudaDeviceSynchronize();
    int hD[M * N];
    cudaMemcpy(hD, dD, sizeof hD, cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int i = 0; i < M * N; ++i) bad += hD[i] != ref[i];
    printf("%-40s %s mismatches=%d  D[0][0..3]=%d %d %d %d ref=%d %d %d %d\n", c.name, cudaGetErrorString(e), bad, hD[0],
           hD[1], hD[2], hD[3], ref[0], ref[1], ref[2], ref[3]);
    if (e != cudaSuccess) return 1;
  }
  return 0;
}
