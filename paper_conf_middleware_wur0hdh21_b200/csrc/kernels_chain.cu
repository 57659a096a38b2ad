// Inference chain: a batch-M (M <= 8) MLP forward  h_{l+1} = act_l(h_l W_l + b_l)  for every
// layer of an inference subgraph, plus the optional softmax head, in ONE persistent kernel —
// the preempter's forward pass whose latency the paper reports (SURVEY.md 8(a) a6,
// PAPER.md:1083-1092, 1213-1220).  Batch 1 makes it a weight stream: 117 MB for the C4 model
// (2048-4096-4096-1000), i.e. HBM-bound, ~18 us at the measured 6.5 TB/s copy rate.
//
// Design (reading Q39): HBM must never idle between layers, and a cold
// 117 MB read needs ~128 KB+ in flight per SM (scripts/read_stream_bench.cu: 16-B loads from all
// threads reach 5.8 TB/s where a single-thread cp.async.bulk ring stays at 4.2-4.7 TB/s).
//   grid     : one CTA per SM, co-resident (cooperative launch); CTA c owns the contiguous
//              float4 range [c U / G, (c+1) U / G) of every layer's row-major W_l
//              (U = K_l N_l / 4): whole rows front to back, the access pattern of a pure copy
//              (a column-block split reads 128-512-B row pieces 16 KB apart).
//   threads  : 512; thread (g, qi) owns column quads q = qi, qi + QT (QT = min(512, Q rounded
//              up to 32)) of rows r = r0 + g, r0 + g + groups, ... (groups = 512 / QT row groups
//              for narrow layers).  Every thread streams its own entries through a private
//              12-row cp.async ring in shared memory (192 KB per SM in flight), and the ring's
//              issue cursor runs ACROSS layer boundaries: while a layer is reduced, the next
//              layer's rows are already in flight.  Row groups are combined in smem in fixed
//              order; the CTA writes its partial row vector part[c][m][:] (global / L2).
//   boundary : grid barrier; each CTA reduces exactly the outputs its rows of layer l + 1 need
//              (its x slice) over the G partials in fixed order, adds the biases (loaded before
//              the layer's stream), applies ReLU, writes them to h_{l+1} — one grid barrier per
//              hidden boundary.  Last layer: CTA c reduces quads [c Q / G, (c+1) Q / G);
//              softmax: per-slice (max, sum exp) published, one more barrier, every CTA
//              normalises its slice with the global pair combined in CTA order.
// Every sum has a fixed order, so repeated launches are bitwise identical (preempted ==
// unpreempted); parity vs the oracle in tests/test_gpu_kernels.py::test_mlp_chain_*.
#include <cuda.h>

#include <algorithm>
#include <atomic>
#include <climits>
#include <cmath>
#include <cstdlib>

#include "sf_device.cuh"
#include "sf_kernels.h"

namespace sfk {
namespace {

constexpr int kThreads = 512;                   // 16 warps, one CTA per SM
constexpr int kMaxQ = 1024;                     // N <= 4096 (two quads per thread at most)
constexpr int kXFloats = 2048;                  // x slice of one layer: M x rows <= 2048
constexpr int kBiasMax = 512;                   // outputs one CTA reduces per layer
constexpr int kGroupF4 = 512;                   // smem row-group combine: groups x M x Q float4
// cp.async ring depth per thread (rows of 2 quads): 12 x 16 KB = 192 KB in flight per SM at
// M <= 2 (the row-group combine buffer grows with M)
constexpr int ring_rows(int MR) { return MR <= 2 ? 12 : 7; }

struct SLayer {
  const float4* W;   // K x N row-major, ld == N
  const float* x;    // M x K (ldx)
  float* y;          // M x N (ldy)
  const float* b0;
  const float* b1;
  const float* b2;
  int K, N, Q, ldx, ldy, relu;  // Q = N / 4
  int U;                        // K * Q float4 units (< 2^31)
};

struct SParams {
  SLayer L[kChainMaxLayers];
  int nl, M;
  float4* part;        // [G][M][Qmax] partial row vectors
  int qmax;
  float* stats;        // [G][M][2] softmax (max, sum of exp) per CTA slice
  unsigned* cnt;       // [0] barrier arrivals, [1] exits (reset by the last CTA out)
  int softmax, sm_ldo;
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

// Grid barrier: the b-th barrier of a launch completes when the arrival counter reaches b * G.
__device__ __forceinline__ void grid_barrier(unsigned* cnt, unsigned target, int tid) {
  __syncthreads();
  if (tid == 0) {
    // release-add (orders this CTA's prior global writes, seen through the bar.sync above)
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" :: "l"(cnt) : "memory");
    while (ld_acquire(cnt) < target) {
    }
  }
  __syncthreads();
}

__device__ __forceinline__ int unit_lo(int U, int c, int G) {
  return static_cast<int>(static_cast<long long>(U) * c / G);
}

// L2 prefetch of [p, p + bytes) in 64 KB bulk pieces (one thread, no completion tracking): a
// CTA whose stream finished early keeps HBM busy with its next layer while slower CTAs finish.
__device__ __forceinline__ void prefetch_l2(const void* p, long long bytes) {
  const char* c = static_cast<const char*>(p);
  for (long long o = 0; o < bytes; o += 65536) {
    const long long n = bytes - o < 65536 ? bytes - o : 65536;
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(c + o), "r"(static_cast<uint32_t>(n))
                 : "memory");
  }
}

// Fixed-order sum over the G partials of one float4 (16 lanes stride the partials, each sums
// its share in order, then a fixed butterfly over the 16 lanes): every CTA that reduces the
// same quad gets the same bits.
template <typename LoadF>
__device__ __forceinline__ float4 sum16(int G, int l16, LoadF ld) {
  float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int base = 0; base < G; base += 160) {
    float4 v[10];
#pragma unroll
    for (int j = 0; j < 10; ++j) {
      const int cc = base + l16 + 16 * j;
      v[j] = cc < G ? ld(cc) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
#pragma unroll
    for (int j = 0; j < 10; ++j) { t.x += v[j].x; t.y += v[j].y; t.z += v[j].z; t.w += v[j].w; }
  }
#pragma unroll
  for (int o = 8; o > 0; o >>= 1) {
    t.x += __shfl_xor_sync(0xffffffffu, t.x, o, 16);
    t.y += __shfl_xor_sync(0xffffffffu, t.y, o, 16);
    t.z += __shfl_xor_sync(0xffffffffu, t.z, o, 16);
    t.w += __shfl_xor_sync(0xffffffffu, t.w, o, 16);
  }
  return t;
}

__device__ __forceinline__ float comp(const float4& v, int j) {
  return j == 0 ? v.x : j == 1 ? v.y : j == 2 ? v.z : v.w;
}

// Per-thread view of one layer: thread (g, qi) owns quads qi, qi + QT of the rows
// r_lo + g + groups j (j < nj) of the CTA's float4 range [u0, u1).
struct TLayer {
  int Q, QT, groups, g, qi, u0, u1, r_lo, nrows, nj;
  __device__ void init(const SLayer& L, int c, int G, int tid) {
    Q = L.Q;
    QT = Q > 512 ? 512 : (Q + 31) / 32 * 32;
    groups = kThreads / QT;
    g = tid / QT;
    qi = tid % QT;
    u0 = unit_lo(L.U, c, G);
    u1 = unit_lo(L.U, c + 1, G);
    r_lo = u0 / Q;
    nrows = u1 > u0 ? (u1 - 1) / Q - r_lo + 1 : 0;
    nj = (g < groups && nrows > g) ? (nrows - g + groups - 1) / groups : 0;
  }
};

__device__ __forceinline__ void cp_async16(void* smem_dst, const void* src, bool valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;"
               :: "r"(sfdev::smem_u32(smem_dst)), "l"(src), "r"(valid ? 16 : 0) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" :: "n"(N) : "memory"); }

template <int MR>
__global__ void __launch_bounds__(kThreads, 1) mlp_stream_kernel(const __grid_constant__ SParams p) {
  constexpr int RS = ring_rows(MR);  // row slots of every thread's cp.async ring
  extern __shared__ __align__(16) unsigned char smem[];
  float4* ring = reinterpret_cast<float4*>(smem);                 // [RS][2][kThreads]
  float* xs = reinterpret_cast<float*>(ring + RS * 2 * kThreads);  // [M][rows] this layer's x slice
  float4* gsum = reinterpret_cast<float4*>(xs + kXFloats);        // [groups][M][QT] row-group partials
  __shared__ float s_bias[kBiasMax];  // summed biases of the outputs this CTA reduces

  const int tid = threadIdx.x, c = blockIdx.x, G = gridDim.x, M = p.M;
  const int warp = tid >> 5, lane = tid & 31;
  unsigned bar_n = 0;

  // issue cursor: (layer il, own row ij) — runs up to RS - 1 rows ahead of consumption, across
  // layer boundaries (the next layer's rows stream while this one is reduced)
  int il = 0, ij = 0, iseq = 0;
  TLayer it;
  it.init(p.L[0], c, G, tid);
  auto issue_one = [&]() {
    while (il < p.nl && ij >= it.nj) {
      if (++il < p.nl) it.init(p.L[il], c, G, tid);
      ij = 0;
    }
    if (il < p.nl) {
      const SLayer& L = p.L[il];
      const int rr = it.g + it.groups * ij;
      float4* slot = ring + (iseq % RS) * 2 * kThreads;
#pragma unroll
      for (int i = 0; i < 2; ++i) {
        const int q = it.qi + i * it.QT;
        const int e = (it.r_lo + rr) * it.Q + q;
        if (i == 0 || it.QT == 512) {
          const bool valid = q < it.Q && e >= it.u0 && e < it.u1;
          cp_async16(slot + i * kThreads + tid, valid ? L.W + e : L.W, valid);
        }
      }
      ++ij;
    }
    cp_async_commit();  // one group per step (empty past the end): wait_group stays constant
    ++iseq;
  };
  for (int k = 0; k < RS - 1; ++k) issue_one();

  {  // layer 0's x slice: the request input
    TLayer t0;
    t0.init(p.L[0], c, G, tid);
    const SLayer& L = p.L[0];
    for (int i = tid; i < M * t0.nrows; i += kThreads) {
      const int m = i / t0.nrows, r = i % t0.nrows;
      xs[i] = __ldcg(L.x + static_cast<size_t>(m) * L.ldx + t0.r_lo + r);
    }
  }
  int cseq = 0;  // consumption sequence number (same order as issue)
  for (int l = 0; l < p.nl; ++l) {
    const SLayer& L = p.L[l];
    TLayer t;
    t.init(L, c, G, tid);
    const int Q = t.Q;
    const bool last = l + 1 == p.nl;
    CHAIN_MARK(l, 0);
    // outputs this CTA reduces after the layer (hidden: the next layer's x rows of its slice;
    // last: quads [q0, q1)); their biases are loaded now and land while the stream runs
    int o_lo, o_n;
    if (!last) {
      TLayer tn;
      tn.init(p.L[l + 1], c, G, tid);
      o_lo = tn.r_lo;
      o_n = tn.nrows;
    } else {
      o_lo = 4 * static_cast<int>(static_cast<long long>(Q) * c / G);
      o_n = 4 * static_cast<int>(static_cast<long long>(Q) * (c + 1) / G) - o_lo;
    }
    float bias = 0.f;
    if (tid < o_n) {
      if (L.b0) bias += __ldg(L.b0 + o_lo + tid);
      if (L.b1) bias += __ldg(L.b1 + o_lo + tid);
      if (L.b2) bias += __ldg(L.b2 + o_lo + tid);
    }
    __syncthreads();  // xs of this layer complete
    float4 acc[MR][2];
#pragma unroll
    for (int m = 0; m < MR; ++m) acc[m][0] = acc[m][1] = make_float4(0.f, 0.f, 0.f, 0.f);
    // the next layer's slice (beyond the ring's run-ahead) to L2, from a thread that never
    // arrives on the grid barrier (its release does not wait for the prefetch)
    const bool pf_thread = tid == 32 && !last;
    auto prefetch_next = [&]() {
      TLayer tn;
      tn.init(p.L[l + 1], c, G, tid);
      if (tn.u1 > tn.u0) prefetch_l2(p.L[l + 1].W + tn.u0, static_cast<long long>(tn.u1 - tn.u0) * 16);
    };
    if (pf_thread && t.nj == 0) prefetch_next();
    for (int j = 0; j < t.nj; ++j) {
      if (pf_thread && j == t.nj / 2) prefetch_next();
      issue_one();
      cp_async_wait<RS - 1>();  // this thread's row cseq has landed
      const float4* slot = ring + (cseq % RS) * 2 * kThreads;
      const int rr = t.g + t.groups * j;
      float4 w[2];
      w[0] = slot[tid];
      w[1] = t.QT == 512 ? slot[kThreads + tid] : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int m = 0; m < MR; ++m) {
        if (m < M) {
          const float xv = xs[m * t.nrows + rr];
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            acc[m][i].x = fmaf(xv, w[i].x, acc[m][i].x);
            acc[m][i].y = fmaf(xv, w[i].y, acc[m][i].y);
            acc[m][i].z = fmaf(xv, w[i].z, acc[m][i].z);
            acc[m][i].w = fmaf(xv, w[i].w, acc[m][i].w);
          }
        }
      }
      ++cseq;
    }
    CHAIN_MARK(l, 1);
    // row groups combined in fixed order (group 0 first), then the CTA's partial row vector
    const int QT = t.QT, groups = t.groups, g = t.g, qi = t.qi;
    if (groups > 1) {
      if (g < groups && g > 0)
#pragma unroll
        for (int m = 0; m < MR; ++m)
          if (m < M) gsum[(g * M + m) * QT + qi] = acc[m][0];
      __syncthreads();
      if (g == 0)
        for (int gg = 1; gg < groups; ++gg)
#pragma unroll
          for (int m = 0; m < MR; ++m)
            if (m < M) {
              const float4 v = gsum[(gg * M + m) * QT + qi];
              acc[m][0].x += v.x; acc[m][0].y += v.y; acc[m][0].z += v.z; acc[m][0].w += v.w;
            }
    }
    if (g == 0) {
#pragma unroll
      for (int i = 0; i < 2; ++i) {
        const int q = qi + i * QT;
        if (q < Q && (i == 0 || QT == 512))
#pragma unroll
          for (int m = 0; m < MR; ++m)
            if (m < M) p.part[(static_cast<size_t>(c) * M + m) * p.qmax + q] = acc[m][i];
      }
    }
    if (tid < o_n) s_bias[tid] = bias;
    grid_barrier(p.cnt, ++bar_n * G, tid);
    CHAIN_MARK(l, 2);
    const int l16 = lane & 15, half = warp * 2 + (lane >> 4);  // 32 half-warps of 16 lanes
    const size_t pstride = static_cast<size_t>(M) * p.qmax;    // float4 between CTAs' partials
    if (!last) {
      // hidden layer: reduce the quads covering exactly the outputs this CTA's rows of layer
      // l + 1 need (its x slice); write them to xs and h_{l+1} (a value two CTAs share is
      // written twice with the same bits)
      const int qa = o_lo / 4, qb = o_n ? (o_lo + o_n - 1) / 4 : qa - 1;
      const int np = M * (qb - qa + 1);
      for (int p0 = 0; p0 < np; p0 += kThreads / 16) {  // uniform trip count (shuffles)
        const int pr = p0 + half;
        const bool on = pr < np;
        const int m = on ? pr / (qb - qa + 1) : 0, q = on ? qa + pr % (qb - qa + 1) : qa;
        const float4* base = p.part + static_cast<size_t>(m) * p.qmax + q;
        const float4 t = sum16(on ? G : 0, l16, [&](int cc) { return __ldcg(base + cc * pstride); });
        if (on && l16 < 4) {
          const int n = 4 * q + l16;
          if (n >= o_lo && n < o_lo + o_n) {
            float v = comp(t, l16) + s_bias[n - o_lo];
            if (L.relu) v = fmaxf(v, 0.f);
            xs[m * o_n + (n - o_lo)] = v;  // next layer's x slice (read after its __syncthreads)
            L.y[static_cast<size_t>(m) * L.ldy + n] = v;
          }
        }
      }
    } else {
      const int q0 = o_lo / 4, nq = o_n / 4;
      const int np = M * nq;
      for (int p0 = 0; p0 < np; p0 += kThreads / 16) {
        const int pr = p0 + half;
        const bool on = pr < np;
        const int m = on ? pr / nq : 0, q = on ? q0 + pr % nq : q0;
        const float4* base = p.part + static_cast<size_t>(m) * p.qmax + q;
        const float4 t = sum16(on ? G : 0, l16, [&](int cc) { return __ldcg(base + cc * pstride); });
        if (on && l16 < 4) {
          const int n = 4 * q + l16;
          float v = comp(t, l16) + s_bias[n - o_lo];
          if (L.relu) v = fmaxf(v, 0.f);
          L.y[static_cast<size_t>(m) * L.ldy + n] = v;
        }
      }
      if (p.softmax) {
        // the last CTA to publish its logits normalises every row (threadfence-reduction
        // pattern: one ticket instead of a second grid barrier); block reductions in fixed order
        __shared__ unsigned s_last;
        __shared__ float s_wr[kThreads / 32];
        __syncthreads();
        if (tid == 0) {
          unsigned tk;
          asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(tk) : "l"(p.cnt + 2) : "memory");
          s_last = tk == static_cast<unsigned>(G) - 1u;
        }
        __syncthreads();
        if (s_last) {
          const int N = L.N;
          auto block_reduce = [&](float v, bool is_max) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
              const float u = __shfl_xor_sync(0xffffffffu, v, o);
              v = is_max ? fmaxf(v, u) : v + u;
            }
            if (lane == 0) s_wr[warp] = v;
            __syncthreads();
            float t = s_wr[0];
            for (int w = 1; w < kThreads / 32; ++w) t = is_max ? fmaxf(t, s_wr[w]) : t + s_wr[w];
            __syncthreads();
            return t;
          };
          for (int m = 0; m < M; ++m) {
            const float* yr = L.y + static_cast<size_t>(m) * L.ldy;
            float mx = -INFINITY;
            for (int n = tid; n < N; n += kThreads) mx = fmaxf(mx, __ldcg(yr + n));
            mx = block_reduce(mx, true);
            float sm = 0.f;
            for (int n = tid; n < N; n += kThreads) sm += expf(__ldcg(yr + n) - mx);
            sm = block_reduce(sm, false);
            for (int n = tid; n < N; n += kThreads)
              p.sm_out[static_cast<size_t>(m) * p.sm_ldo + n] = expf(__ldcg(yr + n) - mx) / sm;
          }
        }
      }
    }
    CHAIN_MARK(l, 3);
  }
  CHAIN_MARK(p.nl, 7);
  // the last CTA out resets the counters for the next launch (stream order)
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    if (atomicAdd(p.cnt + 1, 1u) == static_cast<unsigned>(G) - 1u) {
      p.cnt[0] = 0u;
      p.cnt[1] = 0u;
      p.cnt[2] = 0u;
      __threadfence();
    }
  }
}

int n_sms() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) n = 0;
  }
  return n;
}

size_t smem_bytes(int MR) {
  return size_t(ring_rows(MR)) * 2 * kThreads * 16 + kXFloats * 4 + size_t(kGroupF4) * MR * 16;
}

template <int MR>
cudaError_t configure_t() {
  static std::atomic<uint64_t> configured{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (!(configured.load() & bit)) {
    cudaError_t e = cudaFuncSetAttribute(mlp_stream_kernel<MR>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         static_cast<int>(smem_bytes(MR)));
    if (e != cudaSuccess) return e;
    configured.fetch_or(bit);
  }
  return cudaSuccess;
}

int mr_of(int M) { return M == 1 ? 1 : M == 2 ? 2 : M <= 4 ? 4 : 8; }

int max_q(const ChainArgs& a) {
  int q = 1;
  for (int l = 0; l < a.n_layers; ++l) q = std::max(q, a.layer[l].N / 4);
  return q;
}

template <int MR>
cudaError_t launch_stream_t(const SParams& p, int G, cudaStream_t st) {
  cudaError_t e = configure_t<MR>();
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(G);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem_bytes(MR);
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;  // grid barriers: all CTAs co-resident
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, mlp_stream_kernel<MR>, p);
}

}  // namespace

namespace {
void* g_chain_trace = nullptr;
}
void set_chain_trace(void* dev_buf) { g_chain_trace = dev_buf; }
void* chain_trace_buffer() { return g_chain_trace; }

uint64_t chain_ws_floats(const ChainArgs& a) {
  const uint64_t G = static_cast<uint64_t>(std::max(n_sms(), 1));
  return G * a.M * max_q(a) * 4 + G * a.M * 2;
}
uint64_t chain_counter_slots(const ChainArgs&) { return 3; }

bool chain_eligible(const ChainArgs& a) {
  auto al = [](const void* ptr) { return reinterpret_cast<uintptr_t>(ptr) % 16 == 0; };
  if (a.n_layers < 1 || a.n_layers > kChainMaxLayers || a.M < 1 || a.M > 8 || n_sms() <= 0) return false;
  const int G = n_sms();
  for (int l = 0; l < a.n_layers; ++l) {
    const ChainLayerArgs& L = a.layer[l];
    if (!L.W || !L.x || !L.y || L.K <= 0 || L.N <= 0 || L.N % 4 || L.N / 4 > kMaxQ || L.ldw != L.N ||
        !al(L.W) || static_cast<long long>(L.K) * (L.N / 4) > INT_MAX / 2)
      return false;
    if (l > 0 && (L.x != a.layer[l - 1].y || L.K != a.layer[l - 1].N)) return false;
    if (!L.b[0] && (L.b[1] || L.b[2])) return false;
    // rows a CTA touches (its float4 range may start and end mid-row)
    const long long U = static_cast<long long>(L.K) * (L.N / 4);
    const long long rows = (U + G - 1) / G / (L.N / 4) + 2;
    if (a.M * rows > kXFloats || rows > kBiasMax) return false;
  }
  if (a.softmax && (!a.sm_out || a.sm_n != a.layer[a.n_layers - 1].N ||
                    a.sm_ldi != a.layer[a.n_layers - 1].ldy))
    return false;
  return true;
}

cudaError_t launch_chain(const ChainArgs& a, cudaStream_t st) {
  if (!chain_eligible(a) || !a.counters || !a.ws) return cudaErrorInvalidValue;
  const int G = n_sms();
  SParams p{};
  p.nl = a.n_layers;
  p.M = a.M;
  p.qmax = max_q(a);
  p.part = reinterpret_cast<float4*>(a.ws);
  p.stats = a.ws + static_cast<size_t>(G) * a.M * p.qmax * 4;
  p.cnt = a.counters;
  for (int l = 0; l < a.n_layers; ++l) {
    const ChainLayerArgs& A = a.layer[l];
    SLayer& L = p.L[l];
    L.W = reinterpret_cast<const float4*>(A.W);
    L.x = A.x; L.y = A.y; L.b0 = A.b[0]; L.b1 = A.b[1]; L.b2 = A.b[2];
    L.K = A.K; L.N = A.N; L.Q = A.N / 4; L.ldx = A.ldx; L.ldy = A.ldy; L.relu = A.relu ? 1 : 0;
    L.U = A.K * L.Q;
  }
  p.softmax = a.softmax ? 1 : 0;
  p.sm_out = a.sm_out;
  p.sm_ldo = a.sm_ldo;
  p.trace = static_cast<unsigned long long*>(chain_trace_buffer());
  count_launch();
  switch (mr_of(a.M)) {
    case 1: return launch_stream_t<1>(p, G, st);
    case 2: return launch_stream_t<2>(p, G, st);
    case 4: return launch_stream_t<4>(p, G, st);
    default: return launch_stream_t<8>(p, G, st);
  }
}

}  // namespace sfk
