// Batch <= 8 GEMV over CONSTANT weights re-laid out in blocks (the inference layers of SURVEY.md
// 8(a) a6: the preempter's forward pass).  Batch 1 makes a layer a pure
// weight stream, so what bounds it is how fast HBM can be read: scripts/read_stream_bench.cu
// measured 5.8 TB/s for a contiguous 117 MB read with 16-B LDGs (2 x 256 threads per SM, 16
// loads in flight per thread) against 4.2-4.7 TB/s for any cp.async.bulk ring and ~3.9 TB/s for
// the [K][N] column-block TMA GEMV (512-B row pieces 16 KB apart).  Hence (Q39):
//   layout : W [K][N] is copied once (first request of a binding; sf_refresh_constants) into
//            blocks Wb[cb][r] = W[r kper .. (r+1) kper) x [cb BC .. (cb+1) BC), each block
//            contiguous (kper x QW float4, zero-padded), so every CTA reads ONE contiguous range;
//   grid   : column blocks x 8-CTA clusters (rank r = K slice r), >= 2 CTAs per SM;
//   stream : thread t owns quad q = t % QW of rows rg = t / QW + RL j (RL = 256 / QW); 16-B
//            streaming loads, two 8-row batches in flight (software pipelined); the first batch
//            is issued BEFORE griddep_wait(): under programmatic dependent launch a layer's weight
//            stream starts while its predecessor is still reducing;
//   reduce : RL row groups in smem (fixed order), then the 8 ranks over DSMEM in rank order;
//            bias / ReLU epilogue; optional row softmax by the last column block (fixed order).
// Deterministic: every sum has a fixed order (bitwise-identical repeated launches).
#include <cooperative_groups.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdlib>

#include "sf_device.cuh"
#include "sf_kernels.h"
#include "sf_launch.cuh"

namespace sfk {
namespace {

constexpr int kBlkCluster = 8;   // K split = cluster size (wide layers)
constexpr int kBlkThreads = 256;
constexpr int kBlkBatch = 8;     // rows per load batch (two batches in flight)
constexpr int kBlkMaxKper = 4096;
#ifndef SF_GEMV_MINB
#define SF_GEMV_MINB 2  // CTAs per SM the cluster-free batch-1 layers are compiled for: 3 (80
                        // registers, more of the next layer pre-launched under PDL) measured
                        // 45.0 vs 38.8 us request device time (scripts/r2_minb.sh)
#endif

__device__ __forceinline__ float4 ldg_stream(const float4* p) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}
// with an L2 cache policy (createpolicy): evict_last keeps the block in the persisting L2
// set-aside across requests (infer_l2_persist_bytes), evict_first streams it past
__device__ __forceinline__ float4 ldg_stream_hint(const float4* p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
  return v;
}

// Wb[(cb * CL + r) * kper * QW + row * QW + q] = W[(r * kper + row)][4 (cb QW + q) .. + 3]
__global__ void gemv_block_layout_kernel(const float* __restrict__ W, float4* __restrict__ Wb, int K, int N,
                                         int ldw, int kper, int qw, int n_cb, int cl) {
  const long long total = static_cast<long long>(n_cb) * cl * kper * qw;
  for (long long i = blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x; i < total;
       i += static_cast<long long>(gridDim.x) * blockDim.x) {
    const int q = static_cast<int>(i % qw);
    const long long rowg = i / qw;  // (cb * 8 + r) * kper + row
    const int row = static_cast<int>(rowg % kper);
    const long long blk = rowg / kper;
    const int r = static_cast<int>(blk % cl), cb = static_cast<int>(blk / cl);
    const int k = r * kper + row, n = 4 * (cb * qw + q);
    float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
    if (k < K) {
      const float* src = W + static_cast<size_t>(k) * ldw + n;
      if (n + 3 < N) v = *reinterpret_cast<const float4*>(src);
      else {
        if (n < N) v.x = src[0];
        if (n + 1 < N) v.y = src[1];
        if (n + 2 < N) v.z = src[2];
      }
    }
    Wb[i] = v;
  }
}

// CL: CTAs per column block (the K split; a thread-block cluster reducing over DSMEM when
// CL > 1).  CL = 1 (narrow heads, e.g. 4096 x 1000): each CTA owns whole output columns over
// all of K, so no cluster barrier or DSMEM round trip sits at its end (ncu on the C4 head with
// CL = 8: 30% of warp stalls in the cluster barriers); its row groups reduce as a tree.
template <int MR, int QW, int CL>
__global__ void __launch_bounds__(kBlkThreads, CL == 1 && MR == 1 ? SF_GEMV_MINB : 2)
gemv_blk_kernel(const float4* __restrict__ Wb, const float* __restrict__ X, float* __restrict__ Y, int M,
                int N, int K, int ldx, int ldy, int kper, int acc, const float* __restrict__ b1,
                const float* __restrict__ b2, const float* __restrict__ b3, int relu,
                float* __restrict__ sm_out, int sm_ldo, unsigned* __restrict__ sm_counter, int l2h,
                unsigned long long* __restrict__ tr) {
  constexpr int RL = kBlkThreads / QW;  // row groups
  // debug timeline (sf_debug_chain_trace buffer; C4 layer index from the shape): per layer
  // {min start, max start, min after wait, max after wait, min streamed, max streamed, -, max end}
  unsigned long long* tl = tr ? tr + 8 * (K <= 2048 ? 0 : N <= 1024 ? 2 : 1) : nullptr;
  if (tl && threadIdx.x == 0) {
    const unsigned long long t = sfdev::globaltimer();
    atomicMin(&tl[0], t);
    atomicMax(&tl[1], t);
  }
  extern __shared__ __align__(16) unsigned char blk_smem[];
  float* xs = reinterpret_cast<float*>(blk_smem);                       // [MR][kper]
  float4* red = reinterpret_cast<float4*>(xs + MR * kper);              // [RL][QW]
  __shared__ float4 part[MR * QW];

  namespace cg = cooperative_groups;
  const int rank = CL > 1 ? static_cast<int>(cg::this_cluster().block_rank()) : 0;
  const int cb = blockIdx.x / CL;
  const int tid = threadIdx.x, q = tid % QW, rg = tid / QW;
  const float4* blk = Wb + (static_cast<size_t>(cb) * CL + rank) * kper * QW + q;
  const int nrow = kper / RL;  // rows of this thread (kper is a multiple of RL)
  const int nb = (nrow + kBlkBatch - 1) / kBlkBatch;
  float4 wa[kBlkBatch], wb[kBlkBatch];
  const uint64_t pol = l2h ? sfdev::l2_policy(l2h) : 0ull;
  auto load = [&](float4 (&w)[kBlkBatch], int b) {
#pragma unroll
    for (int u = 0; u < kBlkBatch; ++u) {
      const int j = b * kBlkBatch + u;
      const float4* a = blk + static_cast<size_t>(rg + RL * j) * QW;
      w[u] = j >= nrow ? make_float4(0.f, 0.f, 0.f, 0.f) : l2h ? ldg_stream_hint(a, pol) : ldg_stream(a);
    }
  };
  sfdev::griddep_launch();  // the next layer may start streaming its (constant) weights
#ifndef SF_GEMV_NOPRE
  if (nb > 0) load(wa, 0);  // weights never depend on the predecessor: issue before the wait
  sfdev::griddep_wait();    // x is the predecessor's output
#else  // A/B build: no weight load before the predecessor completes
  sfdev::griddep_wait();
  if (nb > 0) load(wa, 0);
#endif
  if (tl && threadIdx.x == 0) {
    const unsigned long long t = sfdev::globaltimer();
    atomicMin(&tl[2], t);
    atomicMax(&tl[3], t);
  }
  const int k0 = rank * kper;
  // x slice -> smem: 16 independent loads per thread in flight before any store (one L2 round
  // trip, not one per element: the CL = 1 head stages all of K)
  for (int i0 = 0; i0 < MR * kper; i0 += kBlkThreads * 16) {
    float v[16];
#pragma unroll
    for (int u = 0; u < 16; ++u) {
      const int i = i0 + tid + u * kBlkThreads, m = i / kper, kk = i % kper;
      v[u] = (i < MR * kper && m < M && k0 + kk < K) ? X[static_cast<size_t>(m) * ldx + k0 + kk] : 0.f;
    }
#pragma unroll
    for (int u = 0; u < 16; ++u) {
      const int i = i0 + tid + u * kBlkThreads;
      if (i < MR * kper) xs[i] = v[u];
    }
  }
  __syncthreads();
  float4 a[MR];
#pragma unroll
  for (int m = 0; m < MR; ++m) a[m] = make_float4(0.f, 0.f, 0.f, 0.f);
  auto fma_batch = [&](const float4 (&w)[kBlkBatch], int b) {
#pragma unroll
    for (int u = 0; u < kBlkBatch; ++u) {
      const int j = b * kBlkBatch + u;
      if (j < nrow) {
        const int row = rg + RL * j;
#pragma unroll
        for (int m = 0; m < MR; ++m) {
          const float xv = xs[m * kper + row];
          a[m].x = fmaf(xv, w[u].x, a[m].x); a[m].y = fmaf(xv, w[u].y, a[m].y);
          a[m].z = fmaf(xv, w[u].z, a[m].z); a[m].w = fmaf(xv, w[u].w, a[m].w);
        }
      }
    }
  };
  for (int b = 0; b < nb; b += 2) {
    if (b + 1 < nb) load(wb, b + 1);
    fma_batch(wa, b);
    if (b + 1 < nb) {
      if (b + 2 < nb) load(wa, b + 2);
      fma_batch(wb, b + 1);
    }
  }
  if (tl && threadIdx.x == 0) {
    const unsigned long long t = sfdev::globaltimer();
    atomicMin(&tl[4], t);
    atomicMax(&tl[5], t);
  }
  // row groups -> quad partials, fixed order (CL > 1: sequential; CL = 1: a tree, RL up to 128)
#pragma unroll
  for (int m = 0; m < MR; ++m) {
    red[rg * QW + q] = a[m];
    __syncthreads();
    if constexpr (CL == 1) {
      for (int sstep = RL / 2; sstep > 0; sstep >>= 1) {
        if (rg < sstep) {
          const float4 v = red[(rg + sstep) * QW + q];
          float4& t = red[rg * QW + q];
          t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
        }
        __syncthreads();
      }
      if (tid < QW) part[m * QW + tid] = red[tid];
    } else if (tid < QW) {
      float4 t = red[tid];
      for (int g = 1; g < RL; ++g) {
        const float4 v = red[g * QW + tid];
        t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
      }
      part[m * QW + tid] = t;
    }
    __syncthreads();
  }
  if constexpr (CL > 1) cg::this_cluster().sync();
  if (rank == 0 && tid < MR * QW) {  // ranks in order, epilogue
    const int m = tid / QW, n = 4 * (cb * QW + tid % QW);
    if (m < M && n < N) {
      float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
      if constexpr (CL > 1) {
        for (int r = 0; r < CL; ++r) {
          const float4 v = cg::this_cluster().map_shared_rank(part, r)[tid];
          t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
        }
      } else {
        t = part[tid];
      }
      float* o = Y + static_cast<size_t>(m) * ldy + n;
      const float r4[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (n + j >= N) break;
        float v = r4[j];
        if (acc) v = o[j] + v;
        if (b1) v += b1[n + j];
        if (b2) v += b2[n + j];
        if (b3) v += b3[n + j];
        if (relu) v = fmaxf(v, 0.f);
        o[j] = v;
      }
    }
  }
  if (sm_out != nullptr && rank == 0) {
    // fused row softmax: the last column block to publish its outputs normalises every row
    __shared__ int sm_last;
    __shared__ float sm_red[kBlkThreads / 32];
    __threadfence();
    __syncthreads();
    if (tid == 0) sm_last = atomicAdd(sm_counter, 1u) == gridDim.x / CL - 1;
    __syncthreads();
    if (sm_last) {
      if (tl && tid == 0) atomicMax(&tl[6], sfdev::globaltimer());
      __threadfence();
      const int lane = tid & 31, warp = tid >> 5;
      __shared__ float sm_s[kBlkThreads / 32];
      constexpr int kReg = 8;  // row values cached per thread (N <= 2048): ONE L2 round trip
      for (int m = 0; m < M; ++m) {
        // one read pass (all loads issued together): running (max, sum of exp) per thread
        // (online softmax), merged over the block in fixed order; then one normalising pass
        const float* yr = Y + static_cast<size_t>(m) * ldy;
        float mx = -INFINITY, sm = 0.f;
        float v[kReg];
        const bool cached = N <= kReg * kBlkThreads;
        if (cached) {
#pragma unroll
          for (int j = 0; j < kReg; ++j) {
            const int n = tid + j * kBlkThreads;
            v[j] = n < N ? __ldcg(yr + n) : -INFINITY;
          }
#pragma unroll
          for (int j = 0; j < kReg; ++j) mx = fmaxf(mx, v[j]);
          if (mx != -INFINITY) {
#pragma unroll
            for (int j = 0; j < kReg; ++j) sm += expf(v[j] - mx);
          }
        } else {
          for (int n = tid; n < N; n += kBlkThreads) {
            const float x = __ldcg(yr + n);
            if (x > mx) { sm = sm * expf(mx - x) + 1.f; mx = x; }
            else sm += expf(x - mx);
          }
        }
        auto merge = [](float& m1, float& s1, float m2, float s2) {
          if (m2 == -INFINITY) return;
          if (m1 == -INFINITY) { m1 = m2; s1 = s2; return; }
          if (m2 > m1) { s1 = s1 * expf(m1 - m2) + s2; m1 = m2; }
          else s1 += s2 * expf(m2 - m1);
        };
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
          const float m2 = __shfl_xor_sync(0xffffffffu, mx, o), s2 = __shfl_xor_sync(0xffffffffu, sm, o);
          merge(mx, sm, m2, s2);
        }
        if (lane == 0) { sm_red[warp] = mx; sm_s[warp] = sm; }
        __syncthreads();
        mx = sm_red[0];
        sm = sm_s[0];
        for (int w = 1; w < kBlkThreads / 32; ++w) merge(mx, sm, sm_red[w], sm_s[w]);
        __syncthreads();
        float* orow = sm_out + static_cast<size_t>(m) * sm_ldo;
        if (cached) {
#pragma unroll
          for (int j = 0; j < kReg; ++j) {
            const int n = tid + j * kBlkThreads;
            if (n < N) orow[n] = expf(v[j] - mx) / sm;
          }
        } else {
          for (int n = tid; n < N; n += kBlkThreads) orow[n] = expf(__ldcg(yr + n) - mx) / sm;
        }
      }
      if (tid == 0) *sm_counter = 0u;
    }
  }
  if constexpr (CL > 1) cg::this_cluster().sync();  // no CTA leaves while a peer reads its smem
  if (tl && threadIdx.x == 0) atomicMax(&tl[7], sfdev::globaltimer());
}

template <int MR, int QW, int CL>
cudaError_t launch_blk_t(const GemmArgs& a, cudaStream_t st) {
  auto kern = gemv_blk_kernel<MR, QW, CL>;
  const int kper = a.blk_kper;
  const size_t smem = static_cast<size_t>(MR) * kper * 4 + static_cast<size_t>(kBlkThreads / QW) * QW * 16;
  static std::atomic<uint64_t> configured{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (!(configured.load() & bit)) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         static_cast<int>(MR * kBlkMaxKper * 4 + kBlkThreads * 16));
    if (e != cudaSuccess) return e;
    configured.fetch_or(bit);
  }
  const int n_cb = (a.N + 4 * QW - 1) / (4 * QW);
  count_launch();
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(n_cb * CL);
  cfg.blockDim = dim3(kBlkThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  int na = 0;
  if (CL > 1) {
    at[na].id = cudaLaunchAttributeClusterDimension;
    at[na].val.clusterDim.x = CL;
    at[na].val.clusterDim.y = 1;
    at[na].val.clusterDim.z = 1;
    ++na;
  }
  if (pdl_enabled()) {
    at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
  }
  cfg.attrs = at;
  cfg.numAttrs = na;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<const float4*>(a.Bblk), a.A, a.C, a.M, a.N, a.K, a.lda,
                            a.ldc, kper, a.acc ? 1 : 0, a.bias[0], a.bias[1], a.bias[2], a.relu ? 1 : 0,
                            a.sm_out, a.sm_ldo, a.sm_counter, a.l2_hint,
                            static_cast<unsigned long long*>(chain_trace_buffer()));
}

template <int QW, int CL>
cudaError_t dispatch_blk_mr(const GemmArgs& a, cudaStream_t st) {
  if (a.M == 1) return launch_blk_t<1, QW, CL>(a, st);
  if (a.M == 2) return launch_blk_t<2, QW, CL>(a, st);
  if (a.M <= 4) return launch_blk_t<4, QW, CL>(a, st);
  return launch_blk_t<8, QW, CL>(a, st);
}

}  // namespace

GemvBlockPlan plan_gemv_block(int M, int N, int K) {
  GemvBlockPlan p{};
  if (M < 1 || M > 8 || N < 4 || N % 4 || K < 1) return p;
  // Cluster-free blocks (CL = 1): 8- or 16-column blocks over all of K, one CTA each, when that
  // gives one wave of 100-296 CTAs (reading Q44).  SF_GEMV_HEAD: 0 never, 1 narrow
  // heads only (N <= 1184, e.g. the C4 4096 x 1000 head), 2 (default) every eligible layer.
  static const int head = std::getenv("SF_GEMV_HEAD") ? std::atoi(std::getenv("SF_GEMV_HEAD")) : 2;
  if (head && K <= kBlkMaxKper && K >= 1024 && (head == 2 || N <= 4 * 2 * 148)) {
    for (int qw : {2, 4}) {
      const int n_cb = (N + 4 * qw - 1) / (4 * qw);
      if (n_cb < 100 || n_cb > 296) continue;
      const int rl = kBlkThreads / qw;
      p.qw = qw;
      p.cl = 1;
      p.kper = (K + rl - 1) / rl * rl;
      p.n_cb = n_cb;
      p.bytes = static_cast<uint64_t>(p.n_cb) * p.kper * p.qw * 16;
      p.ok = p.kper <= kBlkMaxKper;
      return p;
    }
  }
  // ONE wave: the widest block whose grid still covers every SM (two CTAs fit per SM, so
  // 148..296 CTAs run at once; a second wave would re-pay the ramp)
  int qw = 4;
  for (int w : {32, 16, 8})
    if ((N + 4 * w - 1) / (4 * w) * kBlkCluster >= 148) { qw = w; break; }
  const int rl = kBlkThreads / qw;
  int kper = (K + kBlkCluster - 1) / kBlkCluster;
  kper = (kper + rl - 1) / rl * rl;
  if (kper > 2048) return p;
  p.qw = qw;
  p.cl = kBlkCluster;
  p.kper = kper;
  p.n_cb = (N + 4 * qw - 1) / (4 * qw);
  p.bytes = static_cast<uint64_t>(p.n_cb) * kBlkCluster * kper * qw * 16;
  p.ok = true;
  return p;
}

cudaError_t launch_gemv_block_layout(const float* W, void* Wb, int K, int N, int ldw, const GemvBlockPlan& p,
                                     cudaStream_t st) {
  if (!p.ok) return cudaErrorInvalidValue;
  count_launch();
  gemv_block_layout_kernel<<<148 * 8, 256, 0, st>>>(W, static_cast<float4*>(Wb), K, N, ldw, p.kper, p.qw, p.n_cb,
                                                    p.cl);
  return cudaGetLastError();
}

bool gemv_blk_eligible(const GemmArgs& a) {
  return a.Bblk != nullptr && a.M >= 1 && a.M <= 8 && !a.ta && !a.tb && a.N % 4 == 0 && a.blk_kper > 0;
}

cudaError_t launch_gemv_blk(const GemmArgs& a, cudaStream_t st) {
  if (a.blk_cl == 1)
    return a.blk_qw == 2 ? dispatch_blk_mr<2, 1>(a, st) : a.blk_qw == 4 ? dispatch_blk_mr<4, 1>(a, st)
                                                        : cudaErrorInvalidValue;
  switch (a.blk_qw) {
    case 32: return dispatch_blk_mr<32, kBlkCluster>(a, st);
    case 16: return dispatch_blk_mr<16, kBlkCluster>(a, st);
    case 8: return dispatch_blk_mr<8, kBlkCluster>(a, st);
    case 4: return dispatch_blk_mr<4, kBlkCluster>(a, st);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace sfk
