// Subgraph ops other than GEMM, all HBM-bound SIMT kernels:
//   bias + ReLU / identity, ReLU backward fused with the bias-gradient column sum, column
//   sum, softmax-cross-entropy (forward + backward in one pass per row), softmax, and the
//   multi-tensor SGD-momentum / Adam updates (TF MomentumOptimizer / AdamOptimizer,
//   readings Q8-Q10 in DESIGN.md).
// Determinism (needed for "preempted run == unpreempted run" bit-identity across devices):
// every reduction has a fixed split and a fixed order; split partials are combined by the
// last-arriving CTA in index order; no float atomics.
#include <algorithm>
#include <cmath>

#include "sf_device.cuh"
#include "sf_kernels.h"
#include "sf_launch.cuh"

namespace sfk {
namespace {

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// ---- bias + activation ----------------------------------------------------------------
// act: 0 identity, 1 ReLU, 2 GELU (exact erf form, gelu(u) = 0.5 u (1 + erf(u / sqrt 2)));
// pre (optional) receives u = z + biases (the GELU backward reads it).
__device__ __forceinline__ float act_fwd(int act, float v) {
  if (act == 1) return fmaxf(v, 0.f);
  if (act == 2) return 0.5f * v * (1.f + erff(v * 0.70710678118654752f));
  return v;
}
// Backward of the activation given the mask operand m: ReLU (m = h): [m > 0]; GELU (m = u):
// gelu'(u) = Phi(u) + u phi(u).
__device__ __forceinline__ float act_bwd(int mode, float v, float m) {
  if (mode == 1) return m > 0.f ? v : 0.f;
  const float cdf = 0.5f * (1.f + erff(m * 0.70710678118654752f));
  const float pdf = 0.3989422804014327f * expf(-0.5f * m * m);
  return v * (cdf + m * pdf);
}
__device__ __forceinline__ float4 act_bwd4(int mode, float4 v, float4 m) {
  return make_float4(act_bwd(mode, v.x, m.x), act_bwd(mode, v.y, m.y), act_bwd(mode, v.z, m.z),
                     act_bwd(mode, v.w, m.w));
}

__global__ void bias_act_kernel(const float* __restrict__ z, const float* __restrict__ b1,
                                const float* __restrict__ b2, const float* __restrict__ b3,
                                float* __restrict__ h, float* __restrict__ pre, int rows, int cols,
                                int relu, int vec) {
  sfdev::griddep_wait();
  sfdev::griddep_launch();
  const uint64_t total = static_cast<uint64_t>(rows) * cols;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  if (vec) {
    for (uint64_t q = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; q < total / 4;
         q += stride) {
      const int c = static_cast<int>((q * 4) % cols);
      float4 v = reinterpret_cast<const float4*>(z)[q];
      float4 b = *reinterpret_cast<const float4*>(b1 + c);
      v.x += b.x; v.y += b.y; v.z += b.z; v.w += b.w;
      if (b2) { b = *reinterpret_cast<const float4*>(b2 + c); v.x += b.x; v.y += b.y; v.z += b.z; v.w += b.w; }
      if (b3) { b = *reinterpret_cast<const float4*>(b3 + c); v.x += b.x; v.y += b.y; v.z += b.z; v.w += b.w; }
      if (pre) reinterpret_cast<float4*>(pre)[q] = v;
      v.x = act_fwd(relu, v.x); v.y = act_fwd(relu, v.y); v.z = act_fwd(relu, v.z); v.w = act_fwd(relu, v.w);
      reinterpret_cast<float4*>(h)[q] = v;
    }
    return;
  }
  for (uint64_t i = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; i < total;
       i += stride) {
    const int c = static_cast<int>(i % cols);
    float v = z[i] + b1[c];
    if (b2) v += b2[c];
    if (b3) v += b3[c];
    if (pre) pre[i] = v;
    h[i] = act_fwd(relu, v);
  }
}

// ---- column sum (optionally fused with the ReLU backward mask) ------------------------
// Block = 32 columns x 8 row lanes (each warp reads 128 contiguous bytes of a row);
// grid = (column tiles, row splits).  dz (if non-null) receives x * [mask > 0].
struct ColsumPlan { int col_tiles, rsplit, rper; };
ColsumPlan plan_colsum(int rows, int cols) {
  ColsumPlan p;
  p.col_tiles = (cols + 31) / 32;
  int rs = std::max(1, (2 * 148 + p.col_tiles - 1) / p.col_tiles);
  rs = std::min(rs, std::max(1, (rows + 63) / 64));
  p.rper = (rows + rs - 1) / rs;
  p.rsplit = (rows + p.rper - 1) / p.rper;
  return p;
}

__global__ void __launch_bounds__(256)
colsum_kernel(const float* __restrict__ x, const float* __restrict__ mask, float* __restrict__ dz,
              float* __restrict__ s, int rows, int cols, int rper, int rsplit, float* ws,
              unsigned* counters, int mode) {
  const int lane = threadIdx.x & 31, rl = threadIdx.x >> 5;
  const int col = blockIdx.x * 32 + lane;
  const int z = blockIdx.y;
  const int r0 = z * rper, r1 = min(rows, r0 + rper);
  float acc = 0.f;
  if (col < cols) {
    for (int r = r0 + rl; r < r1; r += 8) {
      const size_t i = static_cast<size_t>(r) * cols + col;
      float v = x[i];
      if (mask) {
        v = act_bwd(mode, v, mask[i]);
        dz[i] = v;
      }
      acc += v;
    }
  }
  __shared__ float red[8][33];
  __shared__ int last;
  red[rl][lane] = acc;
  __syncthreads();
  float part = 0.f;
  if (rl == 0) {
#pragma unroll
    for (int j = 0; j < 8; ++j) part += red[j][lane];
  }
  if (rsplit == 1) {
    if (rl == 0 && col < cols) s[col] = part;
    return;
  }
  if (rl == 0 && col < cols) ws[static_cast<size_t>(z) * cols + col] = part;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) last = atomicAdd(&counters[blockIdx.x], 1u) == static_cast<unsigned>(rsplit - 1);
  __syncthreads();
  if (!last) return;
  __threadfence();
  if (rl == 0 && col < cols) {
    float t = 0.f;
    for (int zz = 0; zz < rsplit; ++zz) t += __ldcg(ws + static_cast<size_t>(zz) * cols + col);
    s[col] = t;
  }
  if (threadIdx.x == 0) counters[blockIdx.x] = 0u;
}

// Vectorized column sum (cols % 4 == 0, 16-B aligned): block = 16 column quads x 16 row
// lanes, 4 rows in flight per thread; split partials [rsplit][cols] are combined by the last
// CTA of the column tile in index order (rows lanes in parallel, then a fixed tree).
struct Colsum4Plan { int col_tiles, rsplit, rper; };
Colsum4Plan plan_colsum4(int rows, int cols) {
  Colsum4Plan p;
  p.col_tiles = (cols / 4 + 15) / 16;
  int rs = std::max(1, (2 * 148 + p.col_tiles - 1) / p.col_tiles);
  rs = std::min(rs, std::max(1, (rows + 127) / 128));
  p.rper = (rows + rs - 1) / rs;
  p.rsplit = (rows + p.rper - 1) / p.rper;
  return p;
}

__global__ void __launch_bounds__(256)
colsum4_kernel(const float* __restrict__ x, const float* __restrict__ mask, float* __restrict__ dz,
               float* __restrict__ s, int rows, int cols, int rper, int rsplit, float* ws,
               unsigned* counters, int mode) {
  const int cq = threadIdx.x & 15, rl = threadIdx.x >> 4;
  const int quad = blockIdx.x * 16 + cq;
  const int nq = cols / 4;
  const int z = blockIdx.y;
  const int r0 = z * rper, r1 = min(rows, r0 + rper);
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  if (quad < nq) {
    const float4* x4 = reinterpret_cast<const float4*>(x);
    const float4* m4 = reinterpret_cast<const float4*>(mask);
    float4* d4 = reinterpret_cast<float4*>(dz);
    int r = r0 + rl;
    for (; r + 48 < r1; r += 64) {
      float4 v[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) v[u] = __ldcs(x4 + static_cast<size_t>(r + 16 * u) * nq + quad);
      if (mask) {
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const size_t i = static_cast<size_t>(r + 16 * u) * nq + quad;
          v[u] = act_bwd4(mode, v[u], __ldcs(m4 + i));
          d4[i] = v[u];
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w;
      }
    }
    for (; r < r1; r += 16) {
      const size_t i = static_cast<size_t>(r) * nq + quad;
      float4 v = __ldcs(x4 + i);
      if (mask) {
        v = act_bwd4(mode, v, __ldcs(m4 + i));
        d4[i] = v;
      }
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
  }
  __shared__ float4 red[16][16];
  __shared__ int last;
  red[rl][cq] = acc;
  __syncthreads();
  float4 part = make_float4(0.f, 0.f, 0.f, 0.f);
  if (rl == 0) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      part.x += red[j][cq].x; part.y += red[j][cq].y; part.z += red[j][cq].z; part.w += red[j][cq].w;
    }
  }
  if (rsplit == 1) {
    if (rl == 0 && quad < nq) reinterpret_cast<float4*>(s)[quad] = part;
    return;
  }
  if (rl == 0 && quad < nq) reinterpret_cast<float4*>(ws)[static_cast<size_t>(z) * nq + quad] = part;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) last = atomicAdd(&counters[blockIdx.x], 1u) == static_cast<unsigned>(rsplit - 1);
  __syncthreads();
  if (!last) return;
  __threadfence();
  // 16 row lanes each sum a strided subset of the splits, then a fixed-order combine
  float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
  if (quad < nq)
    for (int zz = rl; zz < rsplit; zz += 16) {
      const float4 v = __ldcg(reinterpret_cast<const float4*>(ws) + static_cast<size_t>(zz) * nq + quad);
      t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
    }
  __syncthreads();
  red[rl][cq] = t;
  __syncthreads();
  if (rl == 0 && quad < nq) {
    float4 u = red[0][cq];
#pragma unroll
    for (int j = 1; j < 16; ++j) {
      u.x += red[j][cq].x; u.y += red[j][cq].y; u.z += red[j][cq].z; u.w += red[j][cq].w;
    }
    reinterpret_cast<float4*>(s)[quad] = u;
  }
  if (threadIdx.x == 0) counters[blockIdx.x] = 0u;
}

// Deterministic loss reduction shared by the softmax-CE kernels: every CTA reduces its
// threads' partial sums in a fixed tree into ws[blockIdx.x]; the last CTA to arrive sums the
// gridDim.x partials (strided per thread, then the same tree) and resets the counter.
__device__ __forceinline__ float block_sum_tree(float v, float* red) {
  red[threadIdx.x] = v;
  __syncthreads();
  for (int o = 128; o > 0; o >>= 1) {
    if (threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
    __syncthreads();
  }
  const float r = red[0];
  __syncthreads();
  return r;
}

__device__ __forceinline__ void loss_reduce(float part, float* ws, unsigned* counter, float* loss,
                                            int rows) {
  __shared__ float red[256];
  __shared__ int last;
  const float b = block_sum_tree(part, red);
  if (threadIdx.x == 0) ws[blockIdx.x] = b;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) last = atomicAdd(counter, 1u) == gridDim.x - 1;
  __syncthreads();
  if (!last) return;
  __threadfence();
  float t = 0.f;
  for (int i = threadIdx.x; i < static_cast<int>(gridDim.x); i += 256) t += __ldcg(ws + i);
  const float tot = block_sum_tree(t, red);
  if (threadIdx.x == 0) {
    *loss = tot / static_cast<float>(rows);
    *counter = 0u;
  }
}

// Softmax-CE for narrow rows (cols % 4 == 0, cols <= 8 L): L lanes per row, each lane keeps
// up to two float4 of the row in registers (one read pass); shuffles within the L-lane group.
template <int L>
__global__ void __launch_bounds__(256)
softmax_ce_narrow_kernel(const float* __restrict__ l, const int32_t* __restrict__ y,
                         float* __restrict__ loss, float* __restrict__ dl, int rows, int cols,
                         float* ws, unsigned* counter) {
  const int lane = threadIdx.x & 31;
  const int sub = lane % L;                       // lane within the row group
  const int groups_per_block = 256 / L;
  const int g0 = blockIdx.x * groups_per_block + threadIdx.x / L;
  const int stride = gridDim.x * groups_per_block;
  const int warp_first = blockIdx.x * groups_per_block + (threadIdx.x >> 5) * (32 / L);
  const int nq = cols / 4;
  const float inv_b = 1.0f / static_cast<float>(rows);
  float part = 0.f;  // this thread's rows' losses, in row order
  // warp-uniform trip count: every lane joins every shuffle; rows past the end are masked
  for (int base = warp_first, row = g0; base < rows; base += stride, row += stride) {
    const bool active = row < rows;
    if (!active) {
      float m = -INFINITY, s = 0.f;
#pragma unroll
      for (int o = L / 2; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
#pragma unroll
      for (int o = L / 2; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      continue;
    }
    const float4* lr = reinterpret_cast<const float4*>(l + static_cast<size_t>(row) * cols);
    float4* dr = reinterpret_cast<float4*>(dl + static_cast<size_t>(row) * cols);
    float4 v[2];
    bool have[2];
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const int q = sub + u * L;
      have[u] = q < nq;
      v[u] = have[u] ? __ldcs(lr + q) : make_float4(-INFINITY, -INFINITY, -INFINITY, -INFINITY);
    }
    float m = fmaxf(fmaxf(fmaxf(v[0].x, v[0].y), fmaxf(v[0].z, v[0].w)),
                    fmaxf(fmaxf(v[1].x, v[1].y), fmaxf(v[1].z, v[1].w)));
#pragma unroll
    for (int o = L / 2; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    float4 e[2];
    float s = 0.f;
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      if (have[u]) {
        e[u] = make_float4(expf(v[u].x - m), expf(v[u].y - m), expf(v[u].z - m), expf(v[u].w - m));
        s += ((e[u].x + e[u].y) + e[u].z) + e[u].w;
      }
    }
#pragma unroll
    for (int o = L / 2; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const int lab = y[row];
    const bool ok = lab >= 0 && lab < cols;
    const float nan = __int_as_float(0x7fffffff);
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      if (!have[u]) continue;
      const int c0 = 4 * (sub + u * L);
      float4 d;
      d.x = ok ? (e[u].x / s - (c0 == lab ? 1.f : 0.f)) * inv_b : nan;
      d.y = ok ? (e[u].y / s - (c0 + 1 == lab ? 1.f : 0.f)) * inv_b : nan;
      d.z = ok ? (e[u].z / s - (c0 + 2 == lab ? 1.f : 0.f)) * inv_b : nan;
      d.w = ok ? (e[u].w / s - (c0 + 3 == lab ? 1.f : 0.f)) * inv_b : nan;
      dr[sub + u * L] = d;
    }
    if (sub == 0) part += ok ? (m + logf(s)) - l[static_cast<size_t>(row) * cols + lab] : nan;
  }
  loss_reduce(part, ws, counter, loss, rows);
}

// ---- softmax cross-entropy: one warp per row ------------------------------------------
__global__ void __launch_bounds__(256)
softmax_ce_kernel(const float* __restrict__ l, const int32_t* __restrict__ y, float* __restrict__ loss,
                  float* __restrict__ dl, int rows, int cols, float* ws, unsigned* counter) {
  const int lane = threadIdx.x & 31;
  const int warps_total = gridDim.x * 8;
  const float inv_b = 1.0f / static_cast<float>(rows);
  float part = 0.f;
  for (int row = blockIdx.x * 8 + (threadIdx.x >> 5); row < rows; row += warps_total) {
    const float* lr = l + static_cast<size_t>(row) * cols;
    float* dr = dl + static_cast<size_t>(row) * cols;
    const int lab = y[row];
    const bool ok = lab >= 0 && lab < cols;
    float m = -INFINITY;
    for (int c = lane; c < cols; c += 32) m = fmaxf(m, lr[c]);
    m = warp_max(m);
    float s = 0.f;
    for (int c = lane; c < cols; c += 32) s += expf(lr[c] - m);
    s = warp_sum(s);
    for (int c = lane; c < cols; c += 32) {
      const float p = expf(lr[c] - m) / s;
      dr[c] = ok ? (p - (c == lab ? 1.f : 0.f)) * inv_b : __int_as_float(0x7fffffff);
    }
    if (lane == 0) part += ok ? (m + logf(s)) - lr[lab] : __int_as_float(0x7fffffff);
  }
  loss_reduce(part, ws, counter, loss, rows);
}

__global__ void __launch_bounds__(256)
softmax_kernel(const float* __restrict__ l, float* __restrict__ p, int rows, int cols) {
  sfdev::griddep_wait();
  sfdev::griddep_launch();
  const int lane = threadIdx.x & 31;
  for (int row = blockIdx.x * 8 + (threadIdx.x >> 5); row < rows; row += gridDim.x * 8) {
    const float* lr = l + static_cast<size_t>(row) * cols;
    float m = -INFINITY;
    for (int c = lane; c < cols; c += 32) m = fmaxf(m, lr[c]);
    m = warp_max(m);
    float s = 0.f;
    for (int c = lane; c < cols; c += 32) s += expf(lr[c] - m);
    s = warp_sum(s);
    for (int c = lane; c < cols; c += 32) p[static_cast<size_t>(row) * cols + c] = expf(lr[c] - m) / s;
  }
}

// Block-per-row softmax for few, wide rows (batch-1 inference head): 256 threads share a row;
// max / sum reduced through shared memory in a fixed tree order.
__global__ void __launch_bounds__(256)
softmax_block_kernel(const float* __restrict__ l, float* __restrict__ p, int cols) {
  sfdev::griddep_wait();
  sfdev::griddep_launch();
  const float* lr = l + static_cast<size_t>(blockIdx.x) * cols;
  float* pr = p + static_cast<size_t>(blockIdx.x) * cols;
  __shared__ float red[8];
  float m = -INFINITY;
  for (int c = threadIdx.x; c < cols; c += 256) m = fmaxf(m, lr[c]);
  m = warp_max(m);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = m;
  __syncthreads();
  m = red[0];
#pragma unroll
  for (int j = 1; j < 8; ++j) m = fmaxf(m, red[j]);
  __syncthreads();
  float s = 0.f;
  for (int c = threadIdx.x; c < cols; c += 256) s += expf(lr[c] - m);
  s = warp_sum(s);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  s = 0.f;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += red[j];
  for (int c = threadIdx.x; c < cols; c += 256) pr[c] = expf(lr[c] - m) / s;
}

// ---- multi-tensor optimizer updates ---------------------------------------------------
// Descriptor ranges are in units of 4-element quads (prefix sums in .begin, sentinel last).
template <class D>
__device__ __forceinline__ int find_first(const D* d, int n, uint64_t q0) {
  int lo = 0, hi = n - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (d[mid].begin <= q0) lo = mid; else hi = mid - 1;
  }
  return lo;
}

__global__ void __launch_bounds__(256)
sgd_kernel(const SgdDesc* __restrict__ d, int n, uint64_t total, uint64_t per_block) {
  const uint64_t q0 = static_cast<uint64_t>(blockIdx.x) * per_block;
  if (q0 >= total) return;
  const uint64_t q1 = min(q0 + per_block, total);
  __shared__ int first;
  if (threadIdx.x == 0) first = find_first(d, n, q0);
  __syncthreads();
  for (int i = first; i < n; ++i) {
    const uint64_t b = d[i].begin, e = d[i + 1].begin;
    if (b >= q1) break;
    if (e <= q0) continue;
    const uint64_t lo = (q0 > b ? q0 : b) - b, hi = (q1 < e ? q1 : e) - b;
    float* w = d[i].w; float* a = d[i].a; const float* g = d[i].g;
    const uint64_t ne = d[i].n;
    const float lr = d[i].lr, mu = d[i].mu;
    for (uint64_t q = lo + threadIdx.x; q < hi; q += 256) {
      const uint64_t e0 = q * 4;
      if (e0 + 4 <= ne) {
        float4 wv = reinterpret_cast<float4*>(w)[q];
        float4 av = reinterpret_cast<float4*>(a)[q];
        const float4 gv = reinterpret_cast<const float4*>(g)[q];
        av.x = fmaf(mu, av.x, gv.x); av.y = fmaf(mu, av.y, gv.y);
        av.z = fmaf(mu, av.z, gv.z); av.w = fmaf(mu, av.w, gv.w);
        wv.x = fmaf(-lr, av.x, wv.x); wv.y = fmaf(-lr, av.y, wv.y);
        wv.z = fmaf(-lr, av.z, wv.z); wv.w = fmaf(-lr, av.w, wv.w);
        reinterpret_cast<float4*>(a)[q] = av;
        reinterpret_cast<float4*>(w)[q] = wv;
      } else {
        for (uint64_t j = e0; j < ne; ++j) {
          const float an = fmaf(mu, a[j], g[j]);
          a[j] = an;
          w[j] = fmaf(-lr, an, w[j]);
        }
      }
    }
  }
}

__device__ __forceinline__ void adam_elem(float& w, float& m, float& v, float g, float b1,
                                          float b2, float eps, float lr_t) {
  m = fmaf(b1, m, (1.f - b1) * g);
  v = fmaf(b2, v, (1.f - b2) * g * g);
  w = w - lr_t * __fdiv_rn(m, __fsqrt_rn(v) + eps);
}

__global__ void __launch_bounds__(256)
adam_kernel(const AdamDesc* __restrict__ d, int n, uint64_t total, uint64_t per_block,
            const int32_t* __restrict__ step) {
  const uint64_t q0 = static_cast<uint64_t>(blockIdx.x) * per_block;
  if (q0 >= total) return;
  const uint64_t q1 = min(q0 + per_block, total);
  __shared__ int first;
  if (threadIdx.x == 0) first = find_first(d, n, q0);
  __syncthreads();
  const double t = static_cast<double>(*step) + 1.0;
  for (int i = first; i < n; ++i) {
    const uint64_t b = d[i].begin, e = d[i + 1].begin;
    if (b >= q1) break;
    if (e <= q0) continue;
    const uint64_t lo = (q0 > b ? q0 : b) - b, hi = (q1 < e ? q1 : e) - b;
    float* w = d[i].w; float* m = d[i].m; float* v = d[i].v; const float* g = d[i].g;
    const uint64_t ne = d[i].n;
    const float b1 = d[i].b1, b2 = d[i].b2, eps = d[i].eps;
    const float lr_t = static_cast<float>(static_cast<double>(d[i].lr) *
                                          sqrt(1.0 - pow(static_cast<double>(b2), t)) /
                                          (1.0 - pow(static_cast<double>(b1), t)));
    for (uint64_t q = lo + threadIdx.x; q < hi; q += 256) {
      const uint64_t e0 = q * 4;
      if (e0 + 4 <= ne) {
        float4 wv = reinterpret_cast<float4*>(w)[q];
        float4 mv = reinterpret_cast<float4*>(m)[q];
        float4 vv = reinterpret_cast<float4*>(v)[q];
        const float4 gv = reinterpret_cast<const float4*>(g)[q];
        adam_elem(wv.x, mv.x, vv.x, gv.x, b1, b2, eps, lr_t);
        adam_elem(wv.y, mv.y, vv.y, gv.y, b1, b2, eps, lr_t);
        adam_elem(wv.z, mv.z, vv.z, gv.z, b1, b2, eps, lr_t);
        adam_elem(wv.w, mv.w, vv.w, gv.w, b1, b2, eps, lr_t);
        reinterpret_cast<float4*>(w)[q] = wv;
        reinterpret_cast<float4*>(m)[q] = mv;
        reinterpret_cast<float4*>(v)[q] = vv;
      } else {
        for (uint64_t j = e0; j < ne; ++j) adam_elem(w[j], m[j], v[j], g[j], b1, b2, eps, lr_t);
      }
    }
  }
}

unsigned grid_for(uint64_t work_items, uint64_t per_item_min, unsigned cap) {
  uint64_t b = (work_items + per_item_min - 1) / per_item_min;
  return static_cast<unsigned>(std::max<uint64_t>(1, std::min<uint64_t>(b, cap)));
}

}  // namespace

cudaError_t launch_bias_act(const float* z, const float* b1, const float* b2, const float* b3,
                            float* h, int rows, int cols, int act, cudaStream_t st, float* pre) {
  const uint64_t total = static_cast<uint64_t>(rows) * cols;
  if (total == 0) return cudaSuccess;
  auto al = [](const void* p) { return p == nullptr || reinterpret_cast<uintptr_t>(p) % 16 == 0; };
  const int vec = (cols % 4 == 0) && al(z) && al(b1) && al(b2) && al(b3) && al(h) && al(pre);
  const unsigned blocks = grid_for(vec ? total / 4 : total, 256 * 4, 148 * 8);
  count_launch();
  return launch_k(bias_act_kernel, dim3(blocks), dim3(256), 0, st, z, b1, b2, b3, h, pre, rows,
                  cols, act, vec);
}

uint64_t colsum_ws_floats(int rows, int cols) {
  ColsumPlan p = plan_colsum(rows, cols);
  Colsum4Plan q = plan_colsum4(rows, cols);
  return std::max<uint64_t>(p.rsplit > 1 ? static_cast<uint64_t>(p.rsplit) * cols : 0,
                            q.rsplit > 1 ? static_cast<uint64_t>(q.rsplit) * cols : 0);
}
uint64_t colsum_counter_slots(int rows, int cols) {
  return std::max(plan_colsum(rows, cols).col_tiles, plan_colsum4(rows, cols).col_tiles);
}

cudaError_t launch_colsum(const float* x, const float* mask, float* dz, float* s, int rows,
                          int cols, float* ws, unsigned* counters, cudaStream_t st, int mode) {
  if (cols <= 0) return cudaSuccess;
  auto al = [](const void* p) { return p == nullptr || reinterpret_cast<uintptr_t>(p) % 16 == 0; };
  if (cols % 4 == 0 && rows > 0 && al(x) && al(mask) && al(dz) && al(s) && al(ws)) {
    Colsum4Plan q = plan_colsum4(rows, cols);
    if (q.rsplit > 1 && (!ws || !counters)) return cudaErrorInvalidValue;
    dim3 grid(q.col_tiles, q.rsplit);
    colsum4_kernel<<<grid, 256, 0, st>>>(x, mask, dz, s, rows, cols, q.rper, q.rsplit, ws, counters,
                                         mode);
    count_launch();
    return cudaGetLastError();
  }
  ColsumPlan p = plan_colsum(rows, std::max(cols, 1));
  if (rows <= 0) {
    p.rsplit = 1;
    p.rper = 0;
  }
  if (p.rsplit > 1 && (!ws || !counters)) return cudaErrorInvalidValue;
  dim3 grid(p.col_tiles, p.rsplit);
  colsum_kernel<<<grid, 256, 0, st>>>(x, mask, dz, s, rows, cols, p.rper, p.rsplit, ws, counters, mode);
  count_launch();
  return cudaGetLastError();
}

uint64_t softmax_ce_ws_floats(int rows) { return 148 * 8; }  // one partial per CTA (grid cap)

cudaError_t launch_softmax_ce(const float* logits, const int32_t* labels, float* loss,
                              float* dlogits, int rows, int cols, float* ws, unsigned* counter,
                              cudaStream_t st) {
  if (rows <= 0) return cudaSuccess;
  if (!ws || !counter) return cudaErrorInvalidValue;
  auto al = [](const void* p) { return reinterpret_cast<uintptr_t>(p) % 16 == 0; };
  if (cols % 4 == 0 && cols <= 256 && al(logits) && al(dlogits)) {
    const int L = cols <= 16 ? 2 : cols <= 32 ? 4 : cols <= 64 ? 8 : cols <= 128 ? 16 : 32;
    const int per_block = 256 / L;
    const unsigned blocks = grid_for(static_cast<uint64_t>(rows), per_block * 4, 148 * 8);
#define SF_SCE(LL) softmax_ce_narrow_kernel<LL><<<blocks, 256, 0, st>>>(logits, labels, loss, dlogits, rows, cols, ws, counter)
    if (L == 2) SF_SCE(2); else if (L == 4) SF_SCE(4); else if (L == 8) SF_SCE(8);
    else if (L == 16) SF_SCE(16); else SF_SCE(32);
#undef SF_SCE
    count_launch();
    return cudaGetLastError();
  }
  const unsigned blocks = grid_for(static_cast<uint64_t>(rows), 8, 148 * 8);
  softmax_ce_kernel<<<blocks, 256, 0, st>>>(logits, labels, loss, dlogits, rows, cols, ws, counter);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_softmax(const float* logits, float* probs, int rows, int cols, cudaStream_t st) {
  if (rows <= 0) return cudaSuccess;
  if (rows <= 64 && cols >= 256) {
    count_launch();
    return launch_k(softmax_block_kernel, dim3(rows), dim3(256), 0, st, logits, probs, cols);
  }
  const unsigned blocks = grid_for(static_cast<uint64_t>(rows), 8, 148 * 8);
  count_launch();
  return launch_k(softmax_kernel, dim3(blocks), dim3(256), 0, st, logits, probs, rows, cols);
}

cudaError_t launch_sgd(const SgdDesc* d, int n, uint64_t total, cudaStream_t st) {
  if (n <= 0 || total == 0) return cudaSuccess;
  const unsigned blocks = grid_for(total, 1024, 148 * 8);
  const uint64_t per_block = (total + blocks - 1) / blocks;
  sgd_kernel<<<blocks, 256, 0, st>>>(d, n, total, per_block);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_adam(const AdamDesc* d, int n, uint64_t total, const int32_t* step,
                        cudaStream_t st) {
  if (n <= 0 || total == 0) return cudaSuccess;
  const unsigned blocks = grid_for(total, 1024, 148 * 8);
  const uint64_t per_block = (total + blocks - 1) / blocks;
  adam_kernel<<<blocks, 256, 0, st>>>(d, n, total, per_block, step);
  count_launch();
  return cudaGetLastError();
}

}  // namespace sfk
