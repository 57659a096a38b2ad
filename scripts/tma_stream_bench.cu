// Micro-benchmark: HBM streaming rate of a row-major K x N fp32 matrix read by TMA boxes of
// different shapes (and contiguous 1-D bulk copies), one CTA per SM with a 5 x 32 KB ring.
// Decides the W layout / box shape of the fused inference chain (kernels_chain.cu).
// Build+run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tsb scripts/tma_stream_bench.cu -lcuda && /tmp/tsb
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

constexpr int kSlotsMax = 7, kSlot = 32768;
__constant__ int kSlotsC;

__device__ __forceinline__ uint32_t su32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

__global__ void __launch_bounds__(64, 1) stream_kernel(const __grid_constant__ CUtensorMap tm, const float* base,
                                                      int mode, int boxc, int boxr, int ncols_boxes,
                                                      int nrows_boxes, long long bytes_1d, float* sink) {
  extern __shared__ __align__(1024) unsigned char sm[];
  const int kSlots = kSlotsC;
  uint64_t* full = reinterpret_cast<uint64_t*>(sm + kSlotsMax * kSlot);
  const int nbox_total = mode == 2 ? static_cast<int>(bytes_1d / kSlot) : ncols_boxes * nrows_boxes;
  const int per = (nbox_total + gridDim.x - 1) / gridDim.x;
  const int b0 = blockIdx.x * per, b1 = min(nbox_total, b0 + per);
  const int box_bytes = mode == 2 ? kSlot : boxc * boxr * 4;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kSlots; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su32(&full[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  float acc = 0.f;
  int c = 0;
  for (int b = b0; b < b1; ++b, ++c) {
    const int s = c % kSlots;
    if (c >= kSlots) {  // consume the box that occupied this slot
      const uint32_t par = ((c / kSlots) - 1) & 1;
      asm volatile("{\n\t.reg .pred p;\n\tW1:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W1;\n\t}"
                   :: "r"(su32(&full[s])), "r"(par) : "memory");
      acc += reinterpret_cast<float*>(sm + s * kSlot)[0];
    }
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su32(&full[s])), "r"(box_bytes) : "memory");
    const uint32_t dst = su32(sm + s * kSlot);
    if (mode == 2) {
      const float* src = base + static_cast<long long>(b) * (kSlot / 4);
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   :: "r"(dst), "l"(src), "r"(kSlot), "r"(su32(&full[s])) : "memory");
    } else {
      // mode 0: column-block-major (all row boxes of a column block, then the next); 1: row-major
      int cb, rb;
      if (mode == 0) { cb = b / nrows_boxes; rb = b % nrows_boxes; }
      else { rb = b / ncols_boxes; cb = b % ncols_boxes; }
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                   :: "r"(dst), "l"(reinterpret_cast<uint64_t>(&tm)), "r"(su32(&full[s])), "r"(cb * boxc), "r"(rb * boxr) : "memory");
    }
  }
  for (int k = max(0, c - kSlots); k < c; ++k) {
    const int s = k % kSlots;
    const uint32_t par = (k / kSlots) & 1;
    asm volatile("{\n\t.reg .pred p;\n\tW2:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W2;\n\t}"
                 :: "r"(su32(&full[s])), "r"(par) : "memory");
    acc += reinterpret_cast<float*>(sm + s * kSlot)[1];
  }
  if (acc == 12345.f) sink[blockIdx.x] = acc;
}

int main(int argc, char** argv) {
  const int K = argc > 1 ? atoi(argv[1]) : 4096, N = 4096;
  float* W;
  float* sink;
  CK(cudaMalloc(&W, size_t(K) * N * 4));
  CK(cudaMalloc(&sink, 4096));
  CK(cudaMemset(W, 0, size_t(K) * N * 4));
  void* fnp = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fnp, cudaEnableDefault, &q));
  auto enc = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fnp);
  const size_t smem = kSlotsMax * kSlot + 64;
  CK(cudaFuncSetAttribute(stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  float* flush;
  CK(cudaMalloc(&flush, 256 << 20));
  struct Cfg { int mode, bc, br; };
  std::vector<Cfg> cfgs = {{1, 128, 64}, {2, 0, 0}};
  const int slots = argc > 2 ? atoi(argv[2]) : 5;
  CK(cudaMemcpyToSymbol(kSlotsC, &slots, 4));
  for (int grid : {sms}) {
    for (auto cf : cfgs) {
      CUtensorMap tm{};
      if (cf.mode != 2) {
        cuuint64_t dims[2] = {(cuuint64_t)N, (cuuint64_t)K};
        cuuint64_t str[1] = {(cuuint64_t)N * 4};
        cuuint32_t box[2] = {(cuuint32_t)cf.bc, (cuuint32_t)cf.br};
        cuuint32_t es[2] = {1, 1};
        if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, W, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
          printf("encode failed\n");
          return 1;
        }
      }
      const int ncb = cf.mode == 2 ? 0 : N / cf.bc, nrb = cf.mode == 2 ? 0 : K / cf.br;
      float best = 1e9f;
      for (int it = 0; it < 6; ++it) {
        CK(cudaMemset(flush, it, 256 << 20));
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        cudaEventRecord(e0);
        stream_kernel<<<grid, 64, smem>>>(tm, W, cf.mode, cf.bc, cf.br, ncb, nrb, (long long)K * N * 4, sink);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        if (it > 0 && ms < best) best = ms;
      }
      printf("grid %3d mode %d box %3dx%3d: %7.2f us  %6.0f GB/s\n", grid, cf.mode, cf.bc, cf.br, best * 1e3,
             K * (double)N * 4 / (best * 1e-3) / 1e9);
    }
  }
  return 0;
}
