// Inference chain: a batch-M (M <= 8) MLP forward  h_{l+1} = act_l(h_l W_l + b_l)  for every
// layer of an inference subgraph, plus the optional softmax head, in ONE persistent kernel —
// the preempter's forward pass whose latency the paper reports (SURVEY.md 8(a) a6,
// PAPER.md:1083-1092, 1213-1220).  Batch 1 makes it a weight stream: 117 MB for the C4 model
// (2048-4096-4096-1000), i.e. HBM-bound, ~18 us at the measured 6.5 TB/s copy rate.
//
// Design (reading Q42): HBM must never idle, and a layer boundary must not
// become a grid-wide wait.  Every hidden width D_l is split into G contiguous slices, slice c
// owned by CTA c (one CTA per SM, co-resident: cooperative launch), and the layers alternate
// between the two ways a GEMV can be split so that a CTA's output slice of one layer is exactly
// the input slice its next layer needs:
//   layer 0  : COLUMN split — CTA c computes the outputs h_0[:, slice c] in full (every CTA
//              reads all of x, a few KB).  The weights come from a transposed copy W_0^T
//              [N_0][K_0] made once per binding (sf_refresh_constants), so each CTA streams ONE
//              contiguous range (its columns, K_0 floats each).  No reduction across CTAs, so
//              no barrier follows layer 0.
//   layer l>0: ROW split — CTA c multiplies its input slice h_{l-1}[:, slice c] by the rows
//              W_l[slice c, :] (contiguous in the row-major weight) and publishes a partial
//              row vector part[c][m][:]; one grid barrier; then CTA c sums the G partials of the
//              outputs of ITS slice of D_l in fixed order (+ bias, ReLU): its input slice of
//              layer l + 1 (a reduce-scatter through L2).  The last layer reduces its slice of
//              output quads; the last CTA to finish (ticket) normalises the softmax rows.
// So the C4 chain has ONE grid barrier inside the stream (after layer 1), and the last layer's
// row slice (~112 KB per CTA) is bulk-copied (cp.async.bulk, mbarrier) into shared memory at
// kernel start, so its bytes stream together with layers 0 and 1 and nothing is read from HBM
// after the barrier.  Streams use 16-B LDGs with 16 loads in flight per thread (two 8-load
// batches, software pipelined; scripts/read_stream_bench.cu: the access pattern that reaches
// 5.8 TB/s on B200), and the first batch of layer 1 is issued before layer 0's outputs are
// combined.
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

constexpr int kThreads = 512;      // 16 warps, one CTA per SM
constexpr int kWarps = kThreads / 32;
constexpr int kMaxQ = 1024;        // row-split layers: N <= 4096 (two quads per thread at most)
constexpr int kSliceMax = 512;     // elements of one CTA's slice of a hidden width
constexpr int kX0Floats = 16384;   // M x K_0 (padded to 4) of the layer-0 input in smem
constexpr int kChunk4 = 256;       // layer-0 item: 32 lanes x 8 float4 = 4 KB of one column
constexpr int kSmemBudget = 220 * 1024;

struct FLayer {
  const float4* W;   // l == 0: W_0^T [N][Kp / 4]; l > 0: W [K][N / 4] row-major
  float* y;          // M x N (ldy)
  const float* b0;
  const float* b1;
  const float* b2;
  int K, N, Q, ldy, relu;
};

struct FParams {
  FLayer L[kChainMaxLayers];
  int nl, M;
  const float* x;      // layer-0 input, M x K_0 (ldx)
  int ldx, kp0;        // kp0 = K_0 rounded up to 4 (the row pitch of W_0^T)
  float4* part;        // [G][M][qmax] partial row vectors
  int qmax;
  unsigned* cnt;       // [0] barrier arrivals, [1] exits (reset by the last CTA out), [2] ticket
  int softmax, sm_ldo;
  float* sm_out;
  int tail;            // the last layer's row slice is bulk-copied into smem at kernel start
  int tail_bytes, items_max, gsum_f4;  // smem carve-up (bytes / counts, max over CTAs)
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

// slice c of a width D split over G CTAs: [D c / G, D (c + 1) / G)
__device__ __forceinline__ int slice_lo(int D, int c, int G) {
  return D * c / G;  // D <= kSliceMax x G: the product fits 32 bits
}

__device__ __forceinline__ float4 ldg_stream(const float4* p) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}

// L2 prefetch of [p, p + bytes) in 64 KB bulk pieces (one thread, no completion tracking).
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

__device__ __forceinline__ void fma4(float4& a, float x, const float4& w) {
  a.x = fmaf(x, w.x, a.x); a.y = fmaf(x, w.y, a.y); a.z = fmaf(x, w.z, a.z); a.w = fmaf(x, w.w, a.w);
}

// Row-split layer, per thread: quads qi (and 512 + qi when Q > 512: "half" 1) of the rows
// g, g + groups, ... of the CTA's row slice.  Item j = (row g + groups (j >> h), half j & h);
// batches of 8 items, two batches in flight.  acc0 / acc1 hold halves 0 / 1.
template <int MR>
struct RowLayer {
  const float4* src;  // first row of the slice (global, or the smem tail)
  bool in_smem;
  int Q, QV, QT, groups, g, qi, h, nitems;
  float4 wa[8], wb[8];
  float4 acc0[MR], acc1[MR];

  __device__ void init(const float4* s, bool sm, int Q_, int nr, int tid) {
    src = s;
    in_smem = sm;
    Q = Q_;
    QV = Q > 512 ? 512 : Q;
    QT = (QV + 31) / 32 * 32;
    groups = kThreads / QT;
    g = tid / QT;
    qi = tid % QT;
    h = Q > 512 ? 1 : 0;
    const int nrow = (g < groups && nr > g) ? (nr - g + groups - 1) / groups : 0;
    nitems = qi < QV ? nrow << h : 0;
#pragma unroll
    for (int m = 0; m < MR; ++m) acc0[m] = acc1[m] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
  __device__ __forceinline__ int row_of(int j) const { return g + groups * (j >> h); }
  __device__ __forceinline__ int quad_of(int j) const { return qi + ((j & h) << 9); }
  __device__ __forceinline__ void load(float4 (&w)[8], int b) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int j = b * 8 + u, q = quad_of(j);
      const bool valid = j < nitems && q < Q;
      const float4* a = src + static_cast<size_t>(row_of(j)) * Q + q;
      w[u] = !valid ? make_float4(0.f, 0.f, 0.f, 0.f) : in_smem ? *a : ldg_stream(a);
    }
  }
  __device__ __forceinline__ void fma(const float4 (&w)[8], int b, const float* hs, int M) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int j = b * 8 + u;
      if (j < nitems && quad_of(j) < Q) {
        const int row = row_of(j);
#pragma unroll
        for (int m = 0; m < MR; ++m) {
          if (m < M) {
            const float xv = hs[m * kSliceMax + row];
            if ((u & 1) && h) fma4(acc1[m], xv, w[u]);
            else fma4(acc0[m], xv, w[u]);
          }
        }
      }
    }
  }
  // wa must hold batch 0 (load(wa, 0)) before run()
  __device__ void run(const float* hs, int M) {
    const int nb = (nitems + 7) / 8;
    for (int b = 0; b < nb; b += 2) {
      if (b + 1 < nb) load(wb, b + 1);
      fma(wa, b, hs, M);
      if (b + 1 < nb) {
        if (b + 2 < nb) load(wa, b + 2);
        fma(wb, b + 1, hs, M);
      }
    }
  }
};

template <int MR>
__global__ void __launch_bounds__(kThreads, 1) mlp_fold_kernel(const __grid_constant__ FParams p) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int tid = threadIdx.x, c = blockIdx.x, G = gridDim.x, M = p.M;
  const int warp = tid >> 5, lane = tid & 31;
  // smem: [tail: last layer's row slice][x0: M x kp0][hs: MR x kSliceMax][ip: items x MR][gsum]
  float4* tail = reinterpret_cast<float4*>(smem);
  float* x0 = reinterpret_cast<float*>(smem + p.tail_bytes);
  float* hs = x0 + M * p.kp0;
  float* ip = hs + MR * kSliceMax;
  float4* gsum = reinterpret_cast<float4*>(ip + ((p.items_max * MR + 3) & ~3));
  __shared__ __align__(8) uint64_t tbar;
  __shared__ float s_bias[kSliceMax];
  unsigned bar_n = 0;
  const int nl = p.nl;
  CHAIN_MARK(0, 0);

  // ---- layer 0: column split over W_0^T
  const FLayer& L0 = p.L[0];
  const int K4 = p.kp0 / 4, nk = (K4 + kChunk4 - 1) / kChunk4;
  const int n0 = slice_lo(L0.N, c, G), ncols = slice_lo(L0.N, c + 1, G) - n0;
  const int items = ncols * nk;
  float4 wa[8], wb[8];
  auto load_item = [&](float4 (&w)[8], int i) {
    const int col = i / nk, kc = i % nk;
    const float4* base = L0.W + static_cast<size_t>(n0 + col) * K4 + kc * kChunk4 + lane;
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int k4 = kc * kChunk4 + lane + 32 * u;
      w[u] = k4 < K4 ? ldg_stream(base + 32 * u) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  };
  const float4* x0v = reinterpret_cast<const float4*>(x0);
  auto compute_item = [&](const float4 (&w)[8], int i) {
    const int kc = i % nk;
#pragma unroll
    for (int m = 0; m < MR; ++m) {
      if (m < M) {
        float s = 0.f;
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const int k4 = kc * kChunk4 + lane + 32 * u;
          if (k4 < K4) {
            const float4 xv = x0v[m * K4 + k4];
            s = fmaf(xv.x, w[u].x, s); s = fmaf(xv.y, w[u].y, s);
            s = fmaf(xv.z, w[u].z, s); s = fmaf(xv.w, w[u].w, s);
          }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        if (lane == 0) ip[i * MR + m] = s;
      }
    }
  };
  // the request input (a few KB) is staged BEFORE any weight byte is requested: issued together
  // with the stream it would queue behind megabytes of weight reads in DRAM (measured: x
  // landed ~5 us into the kernel); alone it costs one DRAM round trip
  for (int i = tid; i < M * p.kp0; i += kThreads) {
    const int m = i / p.kp0, k = i % p.kp0;
    x0[i] = k < L0.K ? __ldg(p.x + static_cast<size_t>(m) * p.ldx + k) : 0.f;
  }
  __syncthreads();
  CHAIN_MARK(0, 2);
  // ---- the last layer's row slice -> smem (bulk copies; lands while layers 0..nl-2 stream)
  const FLayer& LL = p.L[nl - 1];
  const int lr0 = nl > 1 ? slice_lo(LL.K, c, G) : 0, lr1 = nl > 1 ? slice_lo(LL.K, c + 1, G) : 0;
  const uint32_t tail_bytes = (p.tail && nl > 1) ? static_cast<uint32_t>(lr1 - lr0) * LL.Q * 16u : 0u;
  if (tail_bytes && tid == 0) {
    sfdev::mbar_init(&tbar, 1);
    sfdev::mbar_fence_init();
    sfdev::expect_tx(&tbar, tail_bytes);
    const char* src = reinterpret_cast<const char*>(LL.W + static_cast<size_t>(lr0) * LL.Q);
    for (uint32_t o = 0; o < tail_bytes; o += 32768u) {
      const uint32_t n = tail_bytes - o < 32768u ? tail_bytes - o : 32768u;
      sfdev::bulk_load_1d(sfdev::smem_u32(smem) + o, src + o, n, sfdev::smem_u32(&tbar));
    }
  }

  int it = warp;
  if (it < items) load_item(wa, it);
  // layer-0 biases: loaded now, stored to smem only before the combine (a store here would make
  // the next barrier wait for them behind the weight stream)
  float b0v = 0.f;
  if (tid < ncols) {
    if (L0.b0) b0v += __ldg(L0.b0 + n0 + tid);
    if (L0.b1) b0v += __ldg(L0.b1 + n0 + tid);
    if (L0.b2) b0v += __ldg(L0.b2 + n0 + tid);
  }
  __syncthreads();  // the mbarrier init is visible before anyone waits on it
  CHAIN_MARK(0, 1);
  for (; it < items; it += 2 * kWarps) {
    const int it2 = it + kWarps;
    if (it2 < items) load_item(wb, it2);
    compute_item(wa, it);
    if (it2 < items) {
      if (it2 + kWarps < items) load_item(wa, it2 + kWarps);
      compute_item(wb, it2);
    }
  }
  CHAIN_MARK(0, 5);
  // layer 1's first batch before layer 0's outputs are combined (its rows never wait on them)
  RowLayer<MR> rl;
  if (nl > 1) {
    const FLayer& L1 = p.L[1];
    const int r0 = slice_lo(L1.K, c, G), nr = slice_lo(L1.K, c + 1, G) - r0;
    const bool sm = nl == 2 && tail_bytes;
    rl.init(sm ? tail : L1.W + static_cast<size_t>(r0) * L1.Q, sm, L1.Q, nr, tid);
    if (!sm) rl.load(rl.wa, 0);
  }
  if (tid < ncols) s_bias[tid] = b0v;
  __syncthreads();
  CHAIN_MARK(0, 4);
  for (int i = tid; i < M * ncols; i += kThreads) {
    const int m = i / ncols, col = i % ncols;
    float v = 0.f;
    for (int kc = 0; kc < nk; ++kc) v += ip[(col * nk + kc) * MR + m];
    v += s_bias[col];
    if (L0.relu) v = fmaxf(v, 0.f);
    hs[m * kSliceMax + col] = v;
    L0.y[static_cast<size_t>(m) * L0.ldy + n0 + col] = v;
  }
  __syncthreads();

  // ---- layers 1 .. nl-1: row split, partials, barrier, reduce-scatter
  for (int l = 1; l < nl; ++l) {
    const FLayer& L = p.L[l];
    const bool last = l + 1 == nl;
    const bool from_tail = last && tail_bytes;
    if (l > 1) {
      const int r0 = slice_lo(L.K, c, G), nr = slice_lo(L.K, c + 1, G) - r0;
      rl.init(from_tail ? tail : L.W + static_cast<size_t>(r0) * L.Q, from_tail, L.Q, nr, tid);
      if (!from_tail) rl.load(rl.wa, 0);
    }
    CHAIN_MARK(l, 0);
    if (from_tail) {
      sfdev::mbar_wait(&tbar, 0);
      CHAIN_MARK(l, 6);
      rl.load(rl.wa, 0);
    }
    // outputs this CTA reduces after the layer: hidden -> its slice of N (next layer's rows);
    // last -> quads [Q c / G, Q (c + 1) / G)
    int o_lo, o_n;
    if (!last) {
      o_lo = slice_lo(L.N, c, G);
      o_n = slice_lo(L.N, c + 1, G) - o_lo;
    } else {
      o_lo = 4 * slice_lo(L.Q, c, G);
      o_n = 4 * slice_lo(L.Q, c + 1, G) - o_lo;
    }
    float bias = 0.f;
    if (tid < o_n) {
      if (L.b0) bias += __ldg(L.b0 + o_lo + tid);
      if (L.b1) bias += __ldg(L.b1 + o_lo + tid);
      if (L.b2) bias += __ldg(L.b2 + o_lo + tid);
    }
    rl.run(hs, M);
    CHAIN_MARK(l, 1);
    // row groups combined in fixed order (group 0 first), then the CTA's partial row vector
    if (rl.groups > 1) {
      if (rl.g < rl.groups && rl.g > 0)
#pragma unroll
        for (int m = 0; m < MR; ++m)
          if (m < M) gsum[(rl.g * M + m) * rl.QT + rl.qi] = rl.acc0[m];
      __syncthreads();
      if (rl.g == 0)
        for (int gg = 1; gg < rl.groups; ++gg)
#pragma unroll
          for (int m = 0; m < MR; ++m)
            if (m < M) {
              const float4 v = gsum[(gg * M + m) * rl.QT + rl.qi];
              rl.acc0[m].x += v.x; rl.acc0[m].y += v.y; rl.acc0[m].z += v.z; rl.acc0[m].w += v.w;
            }
    }
    if (rl.g == 0 && rl.qi < rl.QV) {
#pragma unroll
      for (int m = 0; m < MR; ++m) {
        if (m < M) {
          float4* pr = p.part + (static_cast<size_t>(c) * M + m) * p.qmax;
          pr[rl.qi] = rl.acc0[m];
          if (rl.h && rl.qi + 512 < L.Q) pr[rl.qi + 512] = rl.acc1[m];
        }
      }
    }
    if (tid < o_n) s_bias[tid] = bias;
    CHAIN_MARK(l, 5);
    // the next streamed layer's slice to L2 while this CTA waits at the barrier
    if (tid == 32 && l + 1 < nl && !(l + 2 == nl && tail_bytes)) {
      const FLayer& Ln = p.L[l + 1];
      const int r0 = slice_lo(Ln.K, c, G), r1 = slice_lo(Ln.K, c + 1, G);
      if (r1 > r0) prefetch_l2(Ln.W + static_cast<size_t>(r0) * Ln.Q, static_cast<long long>(r1 - r0) * Ln.Q * 16);
    }
    grid_barrier(p.cnt, ++bar_n * G, tid);
    CHAIN_MARK(l, 2);
    const int l16 = lane & 15, half = warp * 2 + (lane >> 4);  // 32 half-warps of 16 lanes
    const size_t pstride = static_cast<size_t>(M) * p.qmax;    // float4 between CTAs' partials
    if (!last) {
      // reduce the quads covering this CTA's slice of N (the next layer's rows); write them to
      // hs and h_{l+1} (a value two CTAs share is written twice with the same bits)
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
            hs[m * kSliceMax + (n - o_lo)] = v;  // next layer's x slice
            L.y[static_cast<size_t>(m) * L.ldy + n] = v;
          }
        }
      }
      __syncthreads();
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
    }
    CHAIN_MARK(l, 3);
  }

  // ---- softmax head: the last CTA to publish its logits normalises every row
  if (p.softmax) {
    const FLayer& L = p.L[nl - 1];
    __shared__ unsigned s_last;
    __shared__ float s_wr[kWarps];
    __syncthreads();
    if (tid == 0) {
      __threadfence();
      unsigned tk;
      asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(tk) : "l"(p.cnt + 2) : "memory");
      s_last = tk == static_cast<unsigned>(G) - 1u;
    }
    __syncthreads();
    if (s_last) {
      __threadfence();
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
        for (int w = 1; w < kWarps; ++w) t = is_max ? fmaxf(t, s_wr[w]) : t + s_wr[w];
        __syncthreads();
        return t;
      };
      constexpr int kReg = 8;  // row values cached per thread: ONE L2 round trip when N <= 4096
      for (int m = 0; m < M; ++m) {
        const float* yr = L.y + static_cast<size_t>(m) * L.ldy;
        float* orow = p.sm_out + static_cast<size_t>(m) * p.sm_ldo;
        if (N <= kReg * kThreads) {
          float v[kReg];
#pragma unroll
          for (int j = 0; j < kReg; ++j) {
            const int n = tid + j * kThreads;
            v[j] = n < N ? __ldcg(yr + n) : -INFINITY;
          }
          float mx = -INFINITY;
#pragma unroll
          for (int j = 0; j < kReg; ++j) mx = fmaxf(mx, v[j]);
          mx = block_reduce(mx, true);
          float sm = 0.f;
#pragma unroll
          for (int j = 0; j < kReg; ++j) sm += tid + j * kThreads < N ? expf(v[j] - mx) : 0.f;
          sm = block_reduce(sm, false);
#pragma unroll
          for (int j = 0; j < kReg; ++j) {
            const int n = tid + j * kThreads;
            if (n < N) orow[n] = expf(v[j] - mx) / sm;
          }
        } else {
          float mx = -INFINITY;
          for (int n = tid; n < N; n += kThreads) mx = fmaxf(mx, __ldcg(yr + n));
          mx = block_reduce(mx, true);
          float sm = 0.f;
          for (int n = tid; n < N; n += kThreads) sm += expf(__ldcg(yr + n) - mx);
          sm = block_reduce(sm, false);
          for (int n = tid; n < N; n += kThreads) orow[n] = expf(__ldcg(yr + n) - mx) / sm;
        }
      }
    }
  }
  CHAIN_MARK(nl, 7);
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

// W_0^T [N][kp] (zero-padded K tail) from the row-major W_0 [K][ldw]: tiled transpose through
// smem (coalesced reads and writes); once per binding, off the request path.
__global__ void w0t_layout_kernel(const float* __restrict__ W, float* __restrict__ Wt, int K, int N, int ldw,
                                  int kp) {
  __shared__ float t[32][33];
  const int k0 = blockIdx.y * 32, n0 = blockIdx.x * 32;
  for (int r = threadIdx.y; r < 32; r += 8) {
    const int k = k0 + r, n = n0 + threadIdx.x;
    t[r][threadIdx.x] = (k < K && n < N) ? W[static_cast<size_t>(k) * ldw + n] : 0.f;
  }
  __syncthreads();
  for (int r = threadIdx.y; r < 32; r += 8) {
    const int n = n0 + r, k = k0 + threadIdx.x;
    if (n < N && k < kp) Wt[static_cast<size_t>(n) * kp + k] = t[threadIdx.x][r];
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

int mr_of(int M) { return M == 1 ? 1 : M == 2 ? 2 : M <= 4 ? 4 : 8; }

int kp_of(int K) { return (K + 3) / 4 * 4; }

int max_q(const ChainArgs& a) {
  int q = 1;
  for (int l = 1; l < a.n_layers; ++l) q = std::max(q, a.layer[l].N / 4);
  return q;
}

// smem carve-up of one launch (without the tail when tail == false)
struct Carve {
  int tail_bytes = 0, items_max = 0, gsum_f4 = 0;
  size_t bytes = 0;
};
Carve carve(const ChainArgs& a, int G, bool tail) {
  Carve k;
  const int MR = mr_of(a.M), nl = a.n_layers;
  if (tail && nl > 1) {
    const ChainLayerArgs& L = a.layer[nl - 1];
    k.tail_bytes = (L.K + G - 1) / G * L.N * 4;
  }
  const ChainLayerArgs& L0 = a.layer[0];
  const int nk = (kp_of(L0.K) / 4 + kChunk4 - 1) / kChunk4;
  k.items_max = (L0.N + G - 1) / G * nk;
  for (int l = 1; l < nl; ++l) {
    const int Q = a.layer[l].N / 4;
    if (Q > 512) continue;
    const int QT = (Q + 31) / 32 * 32, groups = kThreads / QT;
    if (groups > 1) k.gsum_f4 = std::max(k.gsum_f4, groups * a.M * QT);
  }
  k.bytes = static_cast<size_t>(k.tail_bytes) + static_cast<size_t>(a.M) * kp_of(L0.K) * 4 +
            static_cast<size_t>(MR) * kSliceMax * 4 + ((static_cast<size_t>(k.items_max) * MR + 3) & ~size_t(3)) * 4 +
            static_cast<size_t>(k.gsum_f4) * 16;
  return k;
}

template <int MR>
cudaError_t launch_fold_t(const FParams& p, int G, size_t smem, cudaStream_t st) {
  static std::atomic<uint64_t> configured{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (!(configured.load() & bit)) {
    cudaError_t e = cudaFuncSetAttribute(mlp_fold_kernel<MR>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         kSmemBudget);
    static const bool carve_max = !(std::getenv("SF_CHAIN_CARVE") && std::getenv("SF_CHAIN_CARVE")[0] == '0');
    if (e == cudaSuccess && carve_max)
      e = cudaFuncSetAttribute(mlp_fold_kernel<MR>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
    configured.fetch_or(bit);
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(G);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;  // grid barrier: all CTAs co-resident
  at[0].val.cooperative = 1;
  // SF_CHAIN_COOP=0: plain launch (measurement only: co-residency then rests on the grid being
  // one CTA per SM on an otherwise idle device)
  static const bool coop = !(std::getenv("SF_CHAIN_COOP") && std::getenv("SF_CHAIN_COOP")[0] == '0');
  cfg.attrs = at;
  cfg.numAttrs = coop ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, mlp_fold_kernel<MR>, p);
}

}  // namespace

namespace {
void* g_chain_trace = nullptr;
}
void set_chain_trace(void* dev_buf) { g_chain_trace = dev_buf; }
void* chain_trace_buffer() { return g_chain_trace; }

uint64_t chain_ws_floats(const ChainArgs& a) {
  const uint64_t G = static_cast<uint64_t>(std::max(n_sms(), 1));
  return G * a.M * max_q(a) * 4;
}
uint64_t chain_counter_slots(const ChainArgs&) { return 3; }

uint64_t chain_w0t_floats(int K, int N) { return static_cast<uint64_t>(N) * kp_of(K); }

cudaError_t launch_chain_w0t_layout(const float* W, int ldw, int K, int N, float* Wt, cudaStream_t st) {
  count_launch();
  w0t_layout_kernel<<<dim3((N + 31) / 32, (kp_of(K) + 31) / 32), dim3(32, 8), 0, st>>>(W, Wt, K, N, ldw,
                                                                                        kp_of(K));
  return cudaGetLastError();
}

bool chain_eligible(const ChainArgs& a) {
  auto al = [](const void* ptr) { return reinterpret_cast<uintptr_t>(ptr) % 16 == 0; };
  if (a.n_layers < 1 || a.n_layers > kChainMaxLayers || a.M < 1 || a.M > 8 || n_sms() <= 0) return false;
  const int G = n_sms();
  const ChainLayerArgs& L0 = a.layer[0];
  if (!L0.x || !L0.y || L0.K <= 0 || L0.N <= 0 || (L0.N + G - 1) / G > kSliceMax ||
      a.M * kp_of(L0.K) > kX0Floats || static_cast<long long>(L0.N) * kp_of(L0.K) > INT_MAX / 2)
    return false;
  for (int l = 0; l < a.n_layers; ++l) {
    const ChainLayerArgs& L = a.layer[l];
    if (!L.b[0] && (L.b[1] || L.b[2])) return false;
    if (l == 0) continue;
    if (!L.W || !L.x || !L.y || L.K <= 0 || L.N <= 0 || L.N % 4 || L.N / 4 > kMaxQ || L.ldw != L.N ||
        !al(L.W) || static_cast<long long>(L.K) * (L.N / 4) > INT_MAX / 2)
      return false;
    if (L.x != a.layer[l - 1].y || L.K != a.layer[l - 1].N) return false;
    if ((L.K + G - 1) / G > kSliceMax || (L.N + G - 1) / G > kSliceMax) return false;
  }
  if (a.softmax && (!a.sm_out || a.sm_n != a.layer[a.n_layers - 1].N ||
                    a.sm_ldi != a.layer[a.n_layers - 1].ldy))
    return false;
  return carve(a, G, false).bytes <= static_cast<size_t>(kSmemBudget);
}

cudaError_t launch_chain(const ChainArgs& a, cudaStream_t st) {
  if (!chain_eligible(a) || !a.counters || !a.ws || !a.w0t || reinterpret_cast<uintptr_t>(a.w0t) % 16)
    return cudaErrorInvalidValue;
  const int G = n_sms();
  static const bool no_tail = std::getenv("SF_CHAIN_TAIL") && std::getenv("SF_CHAIN_TAIL")[0] == '0';
  Carve k = carve(a, G, !no_tail);
  const bool tail = !no_tail && a.n_layers > 1 && k.bytes <= static_cast<size_t>(kSmemBudget);
  if (!tail) k = carve(a, G, false);
  FParams p{};
  p.nl = a.n_layers;
  p.M = a.M;
  p.x = a.layer[0].x;
  p.ldx = a.layer[0].ldx;
  p.kp0 = kp_of(a.layer[0].K);
  p.qmax = max_q(a);
  p.part = reinterpret_cast<float4*>(a.ws);
  p.cnt = a.counters;
  for (int l = 0; l < a.n_layers; ++l) {
    const ChainLayerArgs& A = a.layer[l];
    FLayer& L = p.L[l];
    L.W = reinterpret_cast<const float4*>(l == 0 ? a.w0t : A.W);
    L.y = A.y; L.b0 = A.b[0]; L.b1 = A.b[1]; L.b2 = A.b[2];
    L.K = A.K; L.N = A.N; L.Q = A.N / 4; L.ldy = A.ldy; L.relu = A.relu ? 1 : 0;
  }
  p.softmax = a.softmax ? 1 : 0;
  p.sm_out = a.sm_out;
  p.sm_ldo = a.sm_ldo;
  p.tail = tail ? 1 : 0;
  p.tail_bytes = k.tail_bytes;
  p.items_max = k.items_max;
  p.gsum_f4 = k.gsum_f4;
  p.trace = static_cast<unsigned long long*>(chain_trace_buffer());
  count_launch();
  switch (mr_of(a.M)) {
    case 1: return launch_fold_t<1>(p, G, k.bytes, st);
    case 2: return launch_fold_t<2>(p, G, k.bytes, st);
    case 4: return launch_fold_t<4>(p, G, k.bytes, st);
    default: return launch_fold_t<8>(p, G, k.bytes, st);
  }
}

}  // namespace sfk
