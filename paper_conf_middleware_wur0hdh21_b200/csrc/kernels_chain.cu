// Fused inference chain: a batch-M (M <= 8) MLP forward  h_{l+1} = act_l(h_l W_l + b_l)  for
// every layer of an inference subgraph, plus the optional softmax head, in ONE persistent
// kernel (SURVEY.md 8(a) a6 — the preempter's forward pass whose latency the paper reports,
// PAPER.md:1213-1220).  The chain is HBM-bound on the weights (29.3M params = 117 MB for the
// C4 model); what a kernel per layer loses is the fill / drain and the split-K reduction at
// every layer boundary.
//
//   clusters : 8 CTAs (one per SM) split K: rank r owns rows [r R, (r+1) R) of every W_l, so
//              its slice of h_l is loaded ONCE per layer.  Cluster c owns the 32-column blocks
//              cb = c, c + n_clusters, ... of every layer (equal shares for the C4 model).
//   warp 8   : one thread streams the CTA's {32 cols x <= 256 rows} W boxes of ALL layers back
//              to back with TMA through a 4-slot mbarrier ring (weights never depend on
//              activations: layer l+1's boxes arrive while layer l is being reduced).
//   warp 9   : x loader — waits on layer l-1's done counter (acquire) and copies the CTA's
//              slice of h_l into a double-buffered smem stage.
//   warps 0-7: thread = (row lane 0..31, column quad 0..7); per column block the 32 row lanes
//              are reduced (warp butterfly + smem, fixed order) into a partial kept in SMEM.
//   layer end: one DSMEM exchange per layer (remote mbarrier arrives); rank r then sums quad r
//              of every local column block over the 8 ranks in rank order, adds the biases,
//              applies ReLU, writes h_{l+1} and bumps the layer's done counter (release).  The
//              CTA completing the last layer runs the softmax and re-zeroes the counters.
// Same arithmetic as the GEMV path (fp32 FMA, fixed-order sums), so results are deterministic;
// parity vs the oracle in tests/test_gpu_kernels.py::test_mlp_chain_*.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdlib>

#include "sf_device.cuh"
#include "sf_kernels.h"
#include "sf_launch.cuh"

namespace sfk {
namespace {

constexpr int kCl = 8;                 // CTAs per cluster (the K split)
constexpr int kCbW = 32;               // columns per column block (128-B W rows)
constexpr int kSlotBytes = 32768;      // ring slot = one W box {32 x <= 256}
constexpr int kSlots = 4;              // 128 KB of W in flight per SM (more does not stream faster)
constexpr int kConsumers = 256;
constexpr int kThreads = kConsumers + 64;
constexpr int kXBufFloats = 4096;      // x slice M x R per buffer (2 buffers)
constexpr int kPartF4 = 1024;          // partials [local cb][M][8 quads] per buffer (2 buffers)
constexpr int kRedF4 = 8 * 8 * 8;      // [M][8 warps][8 quads]
constexpr size_t kSmem = size_t(kSlots) * kSlotBytes + 2 * kXBufFloats * 4 + 2 * kPartF4 * 16 +
                         kRedF4 * 16 + 32 * 8;

struct CLayer {
  CUtensorMap tm;  // W: K rows x N cols, box {32, BR}
  const float* x;
  float* y;
  const float* b0;
  const float* b1;
  const float* b2;
  int K, N, ldx, ldy, relu, n_cb, R, BR, nb, box_bytes, vec_x, expect;
};

struct CParams {
  CLayer L[kChainMaxLayers];
  int nl, M, ncl;
  unsigned* cnt;  // [nl] layer-done counters (each active CTA adds 1)
  int softmax, sm_n, sm_ldi, sm_ldo;
  const float* sm_in;
  float* sm_out;
  unsigned long long* trace;  // diagnostics: [cta][layer * 8 + event] globaltimer ns, or null
};

#define CHAIN_MARK(l, ev)                                                                     \
  do {                                                                                         \
    if (p.trace && tid == 0) p.trace[blockIdx.x * 64 + (l) * 8 + (ev)] = sfdev::globaltimer(); \
  } while (0)

__device__ __forceinline__ unsigned ld_acquire(const unsigned* ptr) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ptr) : "memory");
  return v;
}
__device__ __forceinline__ void consumers_sync() { asm volatile("bar.sync 1, 256;" ::: "memory"); }
__device__ __forceinline__ uint32_t cta_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t mapa(uint32_t addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
  return r;
}
__device__ __forceinline__ void arrive_remote(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" :: "r"(cluster_addr) : "memory");
}
__device__ __forceinline__ void wait_cluster(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tLAB_WAIT:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra LAB_WAIT;\n\t}" :: "r"(sfdev::smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ float4 ld_dsmem(uint32_t cluster_addr) {
  float4 v;
  asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(cluster_addr) : "memory");
  return v;
}

__device__ __forceinline__ int n_local(int n_cb, int cl, int ncl) {
  return cl < n_cb ? (n_cb - 1 - cl) / ncl + 1 : 0;
}

template <int MR>
__global__ void __cluster_dims__(kCl, 1, 1) __launch_bounds__(kThreads, 1)
mlp_chain_kernel(const __grid_constant__ CParams p) {
  extern __shared__ __align__(1024) unsigned char smem[];
  float4* ring = reinterpret_cast<float4*>(smem);
  float* xs = reinterpret_cast<float*>(smem + kSlots * kSlotBytes);
  float4* part = reinterpret_cast<float4*>(xs + 2 * kXBufFloats);
  float4* red = part + 2 * kPartF4;
  uint64_t* full = reinterpret_cast<uint64_t*>(red + kRedF4);
  uint64_t* empty = full + kSlots;
  uint64_t* xfull = empty + kSlots;
  uint64_t* xempty = xfull + 2;
  uint64_t* lbar = xempty + 2;  // layer exchange, one arrive per rank
  uint64_t* ebar = lbar + 2;    // exit: peers finished reading my partials
  __shared__ int s_flag;
  __shared__ float s_red[8];

  const int tid = threadIdx.x, M = p.M, ncl = p.ncl;
  const int rank = static_cast<int>(cta_rank()), cl = blockIdx.x / kCl;
  if (tid == 0) {
    for (int s = 0; s < kSlots; ++s) {
      sfdev::mbar_init(&full[s], 1);
      sfdev::mbar_init(&empty[s], kConsumers / 32);
    }
    for (int b = 0; b < 2; ++b) {
      sfdev::mbar_init(&xfull[b], 1);
      sfdev::mbar_init(&xempty[b], kConsumers / 32);
      sfdev::mbar_init(&lbar[b], kCl);
    }
    sfdev::mbar_init(ebar, kCl);
    sfdev::mbar_fence_init();
  }
  // every CTA's barriers exist before any remote arrive
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  sfdev::griddep_launch();
  const int warp = tid >> 5, lane = tid & 31;

  if (warp == 9) {  // ---- x loader ----
    sfdev::griddep_wait();  // layer 0's x is the predecessor's output
    int a = 0;
    for (int l = 0; l < p.nl; ++l) {
      const CLayer& L = p.L[l];
      if (!n_local(L.n_cb, cl, ncl)) continue;
      const int buf = a & 1;
      if (a >= 2) sfdev::mbar_wait(&xempty[buf], ((a >> 1) - 1) & 1);
      if (l > 0 && lane == 0) {
        const unsigned need = static_cast<unsigned>(p.L[l - 1].expect);
        while (ld_acquire(p.cnt + l - 1) < need) { }
      }
      __syncwarp();
      float* xb = xs + buf * kXBufFloats;
      const int R = L.R, r4 = R / 4, k0 = rank * R;
      for (int i0 = lane; i0 < M * r4; i0 += 32 * 4) {
        float4 v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int i = i0 + 32 * u;
          v[u] = make_float4(0.f, 0.f, 0.f, 0.f);
          if (i < M * r4) {
            const int m = i / r4, k = k0 + 4 * (i % r4);
            const float* xr = L.x + static_cast<size_t>(m) * L.ldx;
            if (L.vec_x && k + 3 < L.K) {
              v[u] = __ldcg(reinterpret_cast<const float4*>(xr + k));
            } else {
              if (k < L.K) v[u].x = __ldcg(xr + k);
              if (k + 1 < L.K) v[u].y = __ldcg(xr + k + 1);
              if (k + 2 < L.K) v[u].z = __ldcg(xr + k + 2);
              if (k + 3 < L.K) v[u].w = __ldcg(xr + k + 3);
            }
          }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (i0 + 32 * u < M * r4) reinterpret_cast<float4*>(xb)[i0 + 32 * u] = v[u];
      }
      __syncwarp();
      if (lane == 0) sfdev::mbar_arrive(&xfull[buf]);
      ++a;
    }
  } else if (warp == 8) {  // ---- W producer ----
    if (lane == 0) {
      int c = 0;
      for (int l = 0; l < p.nl; ++l) {
        const CLayer& L = p.L[l];
        const int nloc = n_local(L.n_cb, cl, ncl);
        for (int j = 0; j < nloc; ++j) {
          const int cb = cl + j * ncl;
          for (int b = 0; b < L.nb; ++b, ++c) {
            const int s = c % kSlots;
            if (c >= kSlots) sfdev::mbar_wait(&empty[s], ((c / kSlots) - 1) & 1);
            sfdev::expect_tx(&full[s], L.box_bytes);
            sfdev::tma_load_2d(sfdev::smem_u32(ring) + s * kSlotBytes, &L.tm, sfdev::smem_u32(&full[s]),
                               cb * kCbW, rank * L.R + b * L.BR);
          }
        }
      }
    }
  } else {  // ---- consumers ----
    sfdev::griddep_wait();
    const int q = lane & 7, rlw = lane >> 3, rl = warp * 4 + rlw;
    int c = 0, a = 0;
    for (int l = 0; l < p.nl; ++l) {
      const CLayer& L = p.L[l];
      const int nloc = n_local(L.n_cb, cl, ncl);
      if (!nloc) continue;
      CHAIN_MARK(l, 0);
      const int buf = a & 1;
      sfdev::mbar_wait(&xfull[buf], (a >> 1) & 1);
      CHAIN_MARK(l, 1);
      const float* xb = xs + buf * kXBufFloats;
      float4* pb = part + buf * kPartF4;
      for (int j = 0; j < nloc; ++j) {
        float4 acc[MR];
#pragma unroll
        for (int m = 0; m < MR; ++m) acc[m] = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int b = 0; b < L.nb; ++b, ++c) {
          const int s = c % kSlots;
          sfdev::mbar_wait(&full[s], (c / kSlots) & 1);
          if (j == 0 && b == 0) CHAIN_MARK(l, 3);
          const float4* tile = ring + s * (kSlotBytes / 16);
          const float* xk = xb + b * L.BR;
#pragma unroll 4
          for (int rr = rl; rr < L.BR; rr += 32) {
            const float4 w4 = tile[rr * 8 + q];
#pragma unroll
            for (int m = 0; m < MR; ++m) {
              if (m < M) {
                const float xv = xk[m * L.R + rr];
                acc[m].x = fmaf(xv, w4.x, acc[m].x); acc[m].y = fmaf(xv, w4.y, acc[m].y);
                acc[m].z = fmaf(xv, w4.z, acc[m].z); acc[m].w = fmaf(xv, w4.w, acc[m].w);
              }
            }
          }
          __syncwarp();
          if (lane == 0) sfdev::mbar_arrive(&empty[s]);
        }
        // 32 row lanes -> partial: butterfly over the warp's 4 row lanes, then 8 warps
#pragma unroll
        for (int m = 0; m < MR; ++m) {
          float4 v = acc[m];
#pragma unroll
          for (int o = 8; o <= 16; o <<= 1) {
            v.x += __shfl_xor_sync(0xffffffffu, v.x, o); v.y += __shfl_xor_sync(0xffffffffu, v.y, o);
            v.z += __shfl_xor_sync(0xffffffffu, v.z, o); v.w += __shfl_xor_sync(0xffffffffu, v.w, o);
          }
          if (rlw == 0 && m < M) red[(m * 8 + warp) * 8 + q] = v;
        }
        consumers_sync();
        if (tid < M * 8) {
          const int m = tid >> 3, qq = tid & 7;
          float4 t = red[(m * 8) * 8 + qq];
#pragma unroll
          for (int w2 = 1; w2 < 8; ++w2) {
            const float4 v = red[(m * 8 + w2) * 8 + qq];
            t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
          }
          pb[(j * M + m) * 8 + qq] = t;
        }
        consumers_sync();
      }
      if (lane == 0) sfdev::mbar_arrive(&xempty[buf]);  // this layer's x slice is consumed
      CHAIN_MARK(l, 4);
      // ---- layer exchange inside the cluster (DSMEM) ----
      if (tid == 0) {
        asm volatile("fence.acq_rel.cluster;" ::: "memory");
        const uint32_t lb = sfdev::smem_u32(&lbar[buf]);
        for (int r2 = 0; r2 < kCl; ++r2) arrive_remote(mapa(lb, r2));
      }
      wait_cluster(&lbar[buf], (a >> 1) & 1);
      CHAIN_MARK(l, 5);
      // rank r finalises column quad r of every local column block, summing ranks in order
      bool wrote = false;
      for (int o = tid; o < nloc * M; o += kConsumers) {
        const int j = o / M, m = o % M;
        const uint32_t src = sfdev::smem_u32(&pb[(j * M + m) * 8 + rank]);
        float4 t = ld_dsmem(mapa(src, 0));
#pragma unroll
        for (int r2 = 1; r2 < kCl; ++r2) {
          const float4 v = ld_dsmem(mapa(src, r2));
          t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
        }
        const int n = (cl + j * ncl) * kCbW + 4 * rank;
        const float r4v[4] = {t.x, t.y, t.z, t.w};
        float* yrow = L.y + static_cast<size_t>(m) * L.ldy;
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          if (n + e >= L.N) continue;
          float v = r4v[e];
          if (L.b0) v += L.b0[n + e];
          if (L.b1) v += L.b1[n + e];
          if (L.b2) v += L.b2[n + e];
          if (L.relu) v = fmaxf(v, 0.f);
          yrow[n + e] = v;
        }
        wrote = true;
      }
      if (wrote) __threadfence();
      consumers_sync();
      if (tid == 0) {
        const unsigned d = atomicAdd(p.cnt + l, 1u);
        const bool fin = (l == p.nl - 1) && d == static_cast<unsigned>(L.expect - 1);
        if (fin) __threadfence();
        s_flag = fin;
      }
      consumers_sync();
      CHAIN_MARK(l, 6);
      ++a;
      if (!s_flag) continue;
      // ---- the whole chain is done: softmax head + counter reset (this CTA is last) ----
      if (p.softmax) {
        for (int m = 0; m < M; ++m) {
          const float* lr = p.sm_in + static_cast<size_t>(m) * p.sm_ldi;
          float* pr = p.sm_out + static_cast<size_t>(m) * p.sm_ldo;
          constexpr int kPer = 16;  // rows up to 16 x 256 values stay in registers
          float v[kPer];
          float mx = -INFINITY;
#pragma unroll
          for (int i = 0; i < kPer; ++i) {
            const int jj = tid + i * kConsumers;
            v[i] = jj < p.sm_n ? __ldcg(lr + jj) : -INFINITY;
            mx = fmaxf(mx, v[i]);
          }
          for (int jj = tid + kPer * kConsumers; jj < p.sm_n; jj += kConsumers) mx = fmaxf(mx, __ldcg(lr + jj));
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
          if (lane == 0) s_red[warp] = mx;
          consumers_sync();
          mx = s_red[0];
#pragma unroll
          for (int w2 = 1; w2 < 8; ++w2) mx = fmaxf(mx, s_red[w2]);
          consumers_sync();
          float sum = 0.f;
#pragma unroll
          for (int i = 0; i < kPer; ++i) {
            v[i] = expf(v[i] - mx);  // exp(-inf) = 0 for the padding
            sum += v[i];
          }
          for (int jj = tid + kPer * kConsumers; jj < p.sm_n; jj += kConsumers) sum += expf(__ldcg(lr + jj) - mx);
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
          if (lane == 0) s_red[warp] = sum;
          consumers_sync();
          sum = s_red[0];
#pragma unroll
          for (int w2 = 1; w2 < 8; ++w2) sum += s_red[w2];
          consumers_sync();
#pragma unroll
          for (int i = 0; i < kPer; ++i) {
            const int jj = tid + i * kConsumers;
            if (jj < p.sm_n) pr[jj] = v[i] / sum;
          }
          for (int jj = tid + kPer * kConsumers; jj < p.sm_n; jj += kConsumers) pr[jj] = expf(__ldcg(lr + jj) - mx) / sum;
        }
      }
      if (tid < p.nl) p.cnt[tid] = 0u;
      CHAIN_MARK(l, 7);
    }
    // exit: my partials may still be read by peers until they have finished their last
    // exchange; each rank tells every peer when its own DSMEM reads are done
    consumers_sync();
    if (tid == 0) {
      const uint32_t eb = sfdev::smem_u32(ebar);
      for (int r2 = 0; r2 < kCl; ++r2) arrive_remote(mapa(eb, r2));
    }
    wait_cluster(ebar, 0);
  }
}

int max_clusters(int MR) {
  static int cache[9] = {0};
  if (cache[MR]) return cache[MR];
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(kCl * 64);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = kSmem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = kCl;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  int n = 0;
  cudaError_t e = cudaSuccess;
  if (MR == 1) e = cudaOccupancyMaxActiveClusters(&n, mlp_chain_kernel<1>, &cfg);
  else if (MR == 2) e = cudaOccupancyMaxActiveClusters(&n, mlp_chain_kernel<2>, &cfg);
  else if (MR == 4) e = cudaOccupancyMaxActiveClusters(&n, mlp_chain_kernel<4>, &cfg);
  else e = cudaOccupancyMaxActiveClusters(&n, mlp_chain_kernel<8>, &cfg);
  if (e != cudaSuccess || n <= 0) {
    cudaGetLastError();
    n = 0;
  }
  cache[MR] = n;
  return n;
}

template <int MR>
cudaError_t configure_t() {
  static std::atomic<uint64_t> configured{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (!(configured.load() & bit)) {
    cudaError_t e = cudaFuncSetAttribute(mlp_chain_kernel<MR>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         static_cast<int>(kSmem));
    if (e != cudaSuccess) return e;
    configured.fetch_or(bit);
  }
  return cudaSuccess;
}

int mr_of(int M) { return M == 1 ? 1 : M == 2 ? 2 : M <= 4 ? 4 : 8; }

int clusters_for(int M) {
  const int MR = mr_of(M);
  cudaError_t e = MR == 1 ? configure_t<1>() : MR == 2 ? configure_t<2>() : MR == 4 ? configure_t<4>() : configure_t<8>();
  if (e != cudaSuccess) return 0;
  return std::min(max_clusters(MR), 18);
}

int rows_per_rank(int K) {
  int R = (K + kCl - 1) / kCl;
  return R > 256 ? (R + 255) / 256 * 256 : (R + 31) / 32 * 32;
}

}  // namespace

namespace {
void* g_chain_trace = nullptr;
}
void set_chain_trace(void* dev_buf) { g_chain_trace = dev_buf; }
void* chain_trace_buffer() { return g_chain_trace; }

uint64_t chain_ws_floats(const ChainArgs&) { return 0; }
uint64_t chain_counter_slots(const ChainArgs& a) { return static_cast<uint64_t>(std::max(a.n_layers, 1)); }

bool chain_eligible(const ChainArgs& a) {
  auto al = [](const void* ptr) { return reinterpret_cast<uintptr_t>(ptr) % 16 == 0; };
  if (a.n_layers < 1 || a.n_layers > kChainMaxLayers || a.M < 1 || a.M > 8) return false;
  const int ncl = clusters_for(a.M);
  if (ncl <= 0) return false;
  for (int l = 0; l < a.n_layers; ++l) {
    const ChainLayerArgs& L = a.layer[l];
    if (!L.W || !L.x || !L.y || L.K <= 0 || L.N <= 0 || L.ldw % 4 || !al(L.W)) return false;
    if (l > 0 && (L.x != a.layer[l - 1].y || L.K != a.layer[l - 1].N)) return false;
    if (!L.b[0] && (L.b[1] || L.b[2])) return false;
    if (a.M * rows_per_rank(L.K) > kXBufFloats) return false;
    const int n_cb = (L.N + kCbW - 1) / kCbW;
    if (((n_cb + ncl - 1) / ncl) * a.M * 8 > kPartF4) return false;
  }
  if (a.softmax && (!a.sm_out || a.sm_n <= 0)) return false;
  return true;
}

cudaError_t launch_chain(const ChainArgs& a, cudaStream_t st) {
  if (!chain_eligible(a) || !a.counters) return cudaErrorInvalidValue;
  const int ncl = clusters_for(a.M);
  CParams p{};
  p.nl = a.n_layers;
  p.M = a.M;
  p.ncl = ncl;
  p.cnt = a.counters;
  for (int l = 0; l < a.n_layers; ++l) {
    const ChainLayerArgs& A = a.layer[l];
    CLayer& L = p.L[l];
    L.R = rows_per_rank(A.K);
    L.BR = std::min(256, L.R);
    L.nb = L.R / L.BR;
    L.box_bytes = kCbW * L.BR * 4;
    if (!make_map2d(&L.tm, A.W, A.N, A.K, static_cast<uint64_t>(A.ldw) * 4, kCbW, L.BR, false))
      return cudaErrorInvalidValue;
    L.x = A.x; L.y = A.y; L.b0 = A.b[0]; L.b1 = A.b[1]; L.b2 = A.b[2];
    L.K = A.K; L.N = A.N; L.ldx = A.ldx; L.ldy = A.ldy; L.relu = A.relu ? 1 : 0;
    L.n_cb = (A.N + kCbW - 1) / kCbW;
    L.expect = std::min(ncl, L.n_cb) * kCl;
    L.vec_x = (A.ldx % 4 == 0 && reinterpret_cast<uintptr_t>(A.x) % 16 == 0) ? 1 : 0;
  }
  p.softmax = a.softmax ? 1 : 0;
  p.sm_n = a.sm_n;
  p.sm_ldi = a.sm_ldi;
  p.sm_ldo = a.sm_ldo;
  p.sm_in = a.layer[a.n_layers - 1].y;
  p.sm_out = a.sm_out;
  p.trace = static_cast<unsigned long long*>(chain_trace_buffer());
  count_launch();
  const dim3 grid(ncl * kCl), block(kThreads);
  switch (mr_of(a.M)) {
    case 1: return launch_k(mlp_chain_kernel<1>, grid, block, kSmem, st, p);
    case 2: return launch_k(mlp_chain_kernel<2>, grid, block, kSmem, st, p);
    case 4: return launch_k(mlp_chain_kernel<4>, grid, block, kSmem, st, p);
    default: return launch_k(mlp_chain_kernel<8>, grid, block, kSmem, st, p);
  }
}

}  // namespace sfk
