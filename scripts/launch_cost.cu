// Host cost of kernel launches on B200 (empty kernels): plain <<<>>>, cudaLaunchKernelEx,
// + PDL attribute, + 8-CTA cluster, + 72 KB dynamic smem, cudaEventRecord, cudaGraphLaunch.
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
__global__ void k_empty(int) {}
__global__ void __cluster_dims__(8, 1, 1) k_cluster(int) {}
__global__ void k_smem(int) { extern __shared__ float s[]; if (threadIdx.x == 9999) s[0] = 0; }
template <class F> double per_call_us(F f, int n = 2000) {
  for (int i = 0; i < 50; ++i) f();
  cudaDeviceSynchronize();
  auto t0 = std::chrono::steady_clock::now();
  for (int i = 0; i < n; ++i) f();
  auto t1 = std::chrono::steady_clock::now();
  cudaDeviceSynchronize();
  return std::chrono::duration<double, std::micro>(t1 - t0).count() / n;
}
int main() {
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, 72 * 1024);
  cudaEvent_t ev;
  cudaEventCreate(&ev);
  auto ex = [&](auto kern, dim3 grid, size_t smem, bool pdl) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid; cfg.blockDim = dim3(288); cfg.dynamicSmemBytes = smem; cfg.stream = st;
    cudaLaunchAttribute at[1];
    if (pdl) { at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
               at[0].val.programmaticStreamSerializationAllowed = 1; cfg.attrs = at; cfg.numAttrs = 1; }
    cudaLaunchKernelEx(&cfg, kern, 0);
  };
  printf("{\"chevron_us\": %.2f", per_call_us([&] { k_empty<<<256, 288, 0, st>>>(0); }));
  printf(", \"ex_us\": %.2f", per_call_us([&] { ex(k_empty, dim3(256), 0, false); }));
  printf(", \"ex_pdl_us\": %.2f", per_call_us([&] { ex(k_empty, dim3(256), 0, true); }));
  printf(", \"ex_cluster_us\": %.2f", per_call_us([&] { ex(k_cluster, dim3(256), 0, false); }));
  printf(", \"ex_cluster_pdl_us\": %.2f", per_call_us([&] { ex(k_cluster, dim3(256), 0, true); }));
  printf(", \"ex_smem72k_pdl_us\": %.2f", per_call_us([&] { ex(k_smem, dim3(256), 72 * 1024, true); }));
  printf(", \"event_record_us\": %.2f", per_call_us([&] { cudaEventRecord(ev, st); }));
  cudaGraph_t g; cudaGraphExec_t ge;
  cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
  for (int i = 0; i < 3; ++i) ex(k_cluster, dim3(256), 0, true);
  cudaStreamEndCapture(st, &g);
  cudaGraphInstantiate(&ge, g, 0);
  cudaGraphUpload(ge, st);
  printf(", \"graph3_us\": %.2f", per_call_us([&] { cudaGraphLaunch(ge, st); }));
  // single launch latency: host issue -> kernel observed done (sync), includes GPU execution
  printf(", \"launch_sync_us\": %.2f}\n", per_call_us([&] { ex(k_empty, dim3(1), 0, false); cudaStreamSynchronize(st); }, 500));
  return 0;
}
