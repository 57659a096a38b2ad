// Probe: cost and abort latency of a device-side gate on queued subgraphs.
//
// A training subgraph version is a CUDA graph.  With the gate, the version is
//   gate kernel (reads a host-written abort word, sets the IF handle) -> IF { body }
// so subgraphs queued on the device but not yet started can be aborted after dispatch
// (queued nodes are aborted, dispatched kernels finish).
// Measures, for a body that spins `body_us` on the device:
//   1. per-graph time back to back, plain vs gated (the gate's steady-state cost);
//   2. drain time after an abort request with W graphs queued, plain vs gated.
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o gate_probe gate_probe.cu
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <thread>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { std::printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); std::exit(1); } } while (0)

__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

__global__ void spin_kernel(unsigned ns, int* sink) {
  const unsigned long long t0 = gtime();
  while (gtime() - t0 < ns) {}
  if (threadIdx.x == 0 && blockIdx.x == 0) atomicAdd(sink, 1);
}

__global__ void gate_kernel(cudaGraphConditionalHandle h, const volatile int* abort_word, int* skipped) {
  const int a = *abort_word;
  cudaGraphSetConditional(h, a ? 0u : 1u);
  if (a) atomicAdd(skipped, 1);
}

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main(int argc, char** argv) {
  const int body_us = argc > 1 ? std::atoi(argv[1]) : 10;
  const int W = argc > 2 ? std::atoi(argv[2]) : 4;
  CK(cudaSetDevice(0));
  cudaStream_t s, cap;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
  int *sink, *skipped, *abort_h;
  CK(cudaMalloc(&sink, 4));
  CK(cudaMalloc(&skipped, 4));
  CK(cudaMemset(skipped, 0, 4));
  CK(cudaHostAlloc(&abort_h, 4, cudaHostAllocMapped));
  *abort_h = 0;
  int* abort_d;
  CK(cudaHostGetDevicePointer(&abort_d, abort_h, 0));

  // plain version: one captured kernel on all SMs
  cudaGraph_t gp;
  CK(cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal));
  spin_kernel<<<148, 128, 0, cap>>>(body_us * 1000u, sink);
  CK(cudaStreamEndCapture(cap, &gp));
  cudaGraphExec_t xp;
  CK(cudaGraphInstantiate(&xp, gp, 0));

  // gated version: gate -> IF { body captured into the conditional's body graph }
  cudaGraph_t gg;
  CK(cudaGraphCreate(&gg, 0));
  cudaGraphConditionalHandle h;
  CK(cudaGraphConditionalHandleCreate(&h, gg, 0, cudaGraphCondAssignDefault));
  cudaGraphNode_t gate;
  {
    void* args[] = {&h, &abort_d, &skipped};
    cudaKernelNodeParams kp{};
    kp.func = reinterpret_cast<void*>(gate_kernel);
    kp.gridDim = dim3(1);
    kp.blockDim = dim3(32);
    kp.kernelParams = args;
    CK(cudaGraphAddKernelNode(&gate, gg, nullptr, 0, &kp));
  }
  cudaGraphNodeParams cp{};
  cp.type = cudaGraphNodeTypeConditional;
  cp.conditional.handle = h;
  cp.conditional.type = cudaGraphCondTypeIf;
  cp.conditional.size = 1;
  cudaGraphNode_t cn;
  CK(cudaGraphAddNode(&cn, gg, &gate, 1, &cp));
  cudaGraph_t body = cp.conditional.phGraph_out[0];
  CK(cudaStreamBeginCaptureToGraph(cap, body, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal));
  spin_kernel<<<148, 128, 0, cap>>>(body_us * 1000u, sink);
  cudaGraph_t body_out;
  CK(cudaStreamEndCapture(cap, &body_out));
  cudaGraphExec_t xg;
  CK(cudaGraphInstantiate(&xg, gg, 0));

  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  std::vector<cudaEvent_t> ring(W);
  for (auto& e : ring) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));

  for (int variant = 0; variant < 2; ++variant) {
    cudaGraphExec_t x = variant ? xg : xp;
    // 1. steady state
    for (int i = 0; i < 20; ++i) CK(cudaGraphLaunch(x, s));
    CK(cudaStreamSynchronize(s));
    const int N = 400;
    CK(cudaEventRecord(e0, s));
    for (int i = 0; i < N; ++i) CK(cudaGraphLaunch(x, s));
    CK(cudaEventRecord(e1, s));
    CK(cudaEventSynchronize(e1));
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    std::printf("%s body %d us: %.2f us per graph back to back\n", variant ? "gated" : "plain", body_us,
                ms * 1e3 / N);
    // 2. abort: W graphs queued, request after the first started; drain = request -> last done
    double drain_sum = 0, drain_max = 0;
    const int R = 50;
    for (int r = 0; r < R; ++r) {
      *abort_h = 0;
      CK(cudaStreamSynchronize(s));
      for (int i = 0; i < W; ++i) {
        CK(cudaGraphLaunch(x, s));
        CK(cudaEventRecord(ring[i], s));
      }
      while (cudaEventQuery(ring[0]) == cudaErrorNotReady) {}  // first subgraph done
      const double t0 = now_us();
      if (variant) *abort_h = 1;
      while (cudaEventQuery(ring[W - 1]) == cudaErrorNotReady) {}
      const double d = now_us() - t0;
      drain_sum += d;
      drain_max = std::max(drain_max, d);
    }
    *abort_h = 0;
    std::printf("%s: abort after subgraph 1 of %d: drain mean %.1f us max %.1f us\n",
                variant ? "gated" : "plain", W, drain_sum / R, drain_max);
  }
  int sk = 0;
  CK(cudaMemcpy(&sk, skipped, 4, cudaMemcpyDeviceToHost));
  std::printf("skipped bodies: %d\n", sk);
  return 0;
}
