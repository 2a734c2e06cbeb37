// Probe: tcgen05 kind::tf32 MMAs with A from TMEM, K-major B (GEMM1) and MN-major B (GEMM2),
// exactly the operand layouts the tensor-core update uses.  Exact small-integer data.
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../paper_conf_edbt_jorgensena23_b200/csrc/tc.cuh"
using namespace egg::tc;

constexpr int M = 128, K1 = 32, N1 = 128, N2 = 32;

__global__ void probe(const float* A, const float* B1, const float* P, const float* V, float* S_out, float* O_out, int mode) {
  __shared__ __align__(1024) float b1[N1 * K1];
  __shared__ __align__(1024) float b2[N1 * N2];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  const int t = threadIdx.x, w = t >> 5;
  // B1 K-major: (e, k) at (e/8)*1024 + (k/4)*128 + (e%8)*16 + (k%4)*4 bytes
  for (int i = t; i < N1 * K1; i += blockDim.x) {
    int e = i / K1, k = i % K1;
    b1[((e / 8) * 1024 + (k / 4) * 128 + (e % 8) * 16 + (k % 4) * 4) / 4] = B1[i];
  }
  // B2 MN-major: (n, k=entry) at (n/4)*128 + (k/8)*1024 + (k%8)*16 + (n%4)*4
  for (int i = t; i < N1 * N2; i += blockDim.x) {
    int k = i / N2, n = i % N2;
    if (mode == 0) b2[((n / 4) * 128 + (k / 8) * 1024 + (k % 8) * 16 + (n % 4) * 4) / 4] = V[i];
    else b2[((n / 8) * 4096 + (k / 4) * 128 + (n % 8) * 16 + (k % 4) * 4) / 4] = V[i];
  }
  if (t == 0) {
    bar_init(&bar, 1);
    bar_fence_init();
  }
  if (w == 0) tmem_alloc<256>(&tbase);
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tb = tbase;
  const uint32_t lane_off = (uint32_t)(32 * w) << 16;
  // row t of A -> TMEM cols [0,32)
  {
    uint32_t v[32];
    for (int k = 0; k < 32; ++k) v[k] = __float_as_uint(A[t * K1 + k]);
    st32(tb + lane_off + 0, v);
    wait_st();
  }
  fence_proxy_async();
  fence_before();
  __syncthreads();
  fence_after();
  if (t == 0) {
    const uint32_t id1 = idesc_tf32(128, N1, false);
    for (int s = 0; s < K1 / 8; ++s)
      mma_ts(tb + 32, tb + 8 * s, sdesc(smem_addr(b1) + s * 256, 128, 1024), id1, s > 0);
    mma_commit(&bar);
  }
  bar_wait(&bar, 0);
  fence_after();
  for (int c = 0; c < N1; c += 32) {
    uint32_t v[32];
    ld32(tb + lane_off + 32 + c, v);
    wait_ld();
    for (int j = 0; j < 32; ++j) S_out[t * N1 + c + j] = __uint_as_float(v[j]);
  }
  // P -> cols [32,160)
  for (int c = 0; c < N1; c += 32) {
    uint32_t v[32];
    for (int j = 0; j < 32; ++j) v[j] = __float_as_uint(P[t * N1 + c + j]);
    st32(tb + lane_off + 32 + c, v);
  }
  wait_st();
  fence_before();
  __syncthreads();
  fence_after();
  if (t == 0) {
    const uint32_t id2 = idesc_tf32(128, N2, mode == 0);
    for (int s = 0; s < N1 / 8; ++s) {
      if (mode == 0) mma_ts(tb + 160, tb + 32 + 8 * s, sdesc(smem_addr(b2) + s * 1024, 1024, 128), id2, s > 0);
      else mma_ts(tb + 160, tb + 32 + 8 * s, sdesc(smem_addr(b2) + s * 256, 128, 4096), id2, s > 0);
    }
    if (mode == 2) {
      const uint32_t id1 = idesc_tf32(128, N1, false);
      for (int s = 0; s < K1 / 8; ++s)
        mma_ts(tb + 32, tb + 8 * s, sdesc(smem_addr(b1) + s * 256, 128, 1024), id1, s > 0);
    }
    mma_commit(&bar);
  }
  bar_wait(&bar, 1);
  fence_after();
  {
    uint32_t v[32];
    ld32(tb + lane_off + 160, v);
    wait_ld();
    for (int j = 0; j < 32; ++j) O_out[t * N2 + j] = __uint_as_float(v[j]);
    ld32(tb + lane_off + 32, v);
    wait_ld();
    if (mode == 2) for (int j = 0; j < 32; ++j) S_out[t * N1 + j] = __uint_as_float(v[j]);
  }
  fence_before();
  __syncthreads();
  if (w == 0) tmem_dealloc<256>(tb);
}

int main(int argc, char** argv) {
  std::vector<float> A(M * K1), B1(N1 * K1), P(M * N1), V(N1 * N2), S(M * N1), O(M * N2);
  srand(1);
  for (auto& x : A) x = (float)(rand() % 17 - 8) / 4.f;
  for (auto& x : B1) x = (float)(rand() % 17 - 8) / 8.f;
  for (int i = 0; i < M; ++i)
    for (int j = 0; j < N1; ++j) P[i * N1 + j] = ((i * 7 + j * 3) % 5) < 2 ? 1.f : 0.f;
  for (auto& x : V) x = (float)(rand() % 201 - 100);
  float *dA, *dB1, *dP, *dV, *dS, *dO;
  cudaMalloc(&dA, A.size() * 4); cudaMalloc(&dB1, B1.size() * 4); cudaMalloc(&dP, P.size() * 4);
  cudaMalloc(&dV, V.size() * 4); cudaMalloc(&dS, S.size() * 4); cudaMalloc(&dO, O.size() * 4);
  cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(dB1, B1.data(), B1.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(dP, P.data(), P.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(dV, V.data(), V.size() * 4, cudaMemcpyHostToDevice);
  int mode = argc > 1 ? atoi(argv[1]) : 0;
  probe<<<148, 128>>>(dA, dB1, dP, dV, dS, dO, mode);
  cudaError_t e = cudaDeviceSynchronize();
  printf("kernel: %s\n", cudaGetErrorString(e));
  cudaMemcpy(S.data(), dS, S.size() * 4, cudaMemcpyDeviceToHost);
  cudaMemcpy(O.data(), dO, O.size() * 4, cudaMemcpyDeviceToHost);
  int bad1 = 0, bad2 = 0;
  for (int i = 0; i < M; ++i)
    for (int j = 0; j < N1; ++j) {
      double r = 0;
      for (int k = 0; k < K1; ++k) r += (double)A[i * K1 + k] * B1[j * K1 + k];
      if (r != S[i * N1 + j]) { if (bad1 < 5) printf("S[%d][%d] = %g want %g\n", i, j, S[i * N1 + j], r); ++bad1; }
    }
  for (int i = 0; i < M; ++i)
    for (int n = 0; n < N2; ++n) {
      double r = 0;
      for (int k = 0; k < N1; ++k) r += (double)P[i * N1 + k] * V[k * N2 + n];
      if (r != O[i * N2 + n]) { if (bad2 < 5) printf("O[%d][%d] = %g want %g\n", i, n, O[i * N2 + n], r); ++bad2; }
    }
  printf("GEMM1 mismatches %d / %d, GEMM2 mismatches %d / %d\n", bad1, M * N1, bad2, M * N2);
  return (bad1 || bad2) ? 1 : 0;
}
