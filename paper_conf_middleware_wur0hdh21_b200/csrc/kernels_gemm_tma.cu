// TMA-fed tcgen05 3xTF32 GEMM (the training-subgraph GEMM of SURVEY.md K5, round-2 design).
//
//   warp 0     : TMA producer — one thread loads the raw fp32 A / B tiles of a stage with
//                cp.async.bulk.tensor (SWIZZLE_128B).  K-contiguous operands arrive as the
//                canonical K-major SW128 layout; MN-contiguous operands as MN-major SW128
//                atoms (32 MN x 8 K per 1 KiB atom, 4 KiB per 32-wide MN block).
//   warps 1-8  : converters — split every element in place into tf32 hi (low 13 mantissa
//                bits cleared) and a separate lo = tf32(x - hi) buffer with the same layout
//                (elementwise, layout-agnostic, conflict-free 16-B accesses); warps 1-4 then
//                run the epilogue.
//   warp 9     : TMEM allocation + one elected thread issuing tcgen05.mma.kind::tf32
//                (lo.hi, hi.lo, hi.hi per K=8 step) with K- or MN-major smem descriptors.
//   epilogue   : tcgen05.ld -> registers -> swizzled smem box -> TMA store (rows / columns
//                beyond the matrix are clipped by the tensor map); split-K partials go to a
//                3-D workspace map and the last CTA of a tile sums them in order z=0..S-1.
//
// Same numerics as kernels_gemm.cu (parity-tested), different data movement.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>
#include <atomic>
#include <mutex>

#include "sf_device.cuh"
#include "sf_kernels.h"

namespace sfk {
namespace {

constexpr int BM = 128;
constexpr int BK = 32;
constexpr int kConvWarps = 8;
constexpr int kMmaWarp = 9;
constexpr int kThreads = 10 * 32;

template <int BN>
struct TCfg {
  static constexpr int STAGES = BN == 64 ? 4 : 3;
  static constexpr int A_BYTES = BM * BK * 4;
  static constexpr int B_BYTES = BN * BK * 4;
  static constexpr int STAGE_BYTES = 2 * A_BYTES + 2 * B_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 256;
  static constexpr uint32_t TMEM_COLS = BN;
};

struct TParams {
  int M, N, K, ldc;
  int splits, kb_per_split, acc, dbg;
  float* C;
  float* ws;
  unsigned* counters;
};

__device__ __forceinline__ uint64_t desc_k(uint32_t saddr) {  // K-major SW128
  return static_cast<uint64_t>((saddr & 0x3FFFFu) >> 4) | (1ull << 16) | (64ull << 32) | (1ull << 46) |
         (2ull << 61);
}
__device__ __forceinline__ uint64_t desc_mn(uint32_t saddr) {
  // MN-major 32-bit operands use SWIZZLE_128B_BASE32B (layout type 1; 32-B swizzle atoms,
  // CUTLASS Layout_MN_SW128_32B_Atom): 4-row K groups 512 B apart (SBO), 32-element MN
  // blocks 4096 B apart (LBO).  TMA writes it with CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B.
  return static_cast<uint64_t>((saddr & 0x3FFFFu) >> 4) | (256ull << 16) | (32ull << 32) |
         (1ull << 46) | (1ull << 61);
}

__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* m, uint32_t bar, int x,
                                            int y) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
      :: "r"(dst), "l"(reinterpret_cast<uint64_t>(m)), "r"(bar), "r"(x), "r"(y) : "memory");
}
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* m, uint32_t src, int x, int y) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];"
               :: "l"(reinterpret_cast<uint64_t>(m)), "r"(src), "r"(x), "r"(y) : "memory");
}
__device__ __forceinline__ void tma_store_3d(const CUtensorMap* m, uint32_t src, int x, int y, int z) {
  asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];"
               :: "l"(reinterpret_cast<uint64_t>(m)), "r"(src), "r"(x), "r"(y), "r"(z) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read1() {
  asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;"
               :: "r"(sfdev::smem_u32(bar)), "r"(bytes) : "memory");
}

__device__ __forceinline__ float tf32_trunc(float x) {
  return __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
}

// Split NQ float4 of a tile (thread stride 256): lo = tf32(x - trunc_tf32(x)) into `lo`;
// unless RAW_HI, also overwrite x with trunc_tf32(x).  All loads are issued first.
template <int NQ, bool RAW_HI>
__device__ __forceinline__ void split_tile(float4* __restrict__ x, float4* __restrict__ lo, int t) {
  float4 v[NQ];
#pragma unroll
  for (int i = 0; i < NQ; ++i) v[i] = x[t + 256 * i];
#pragma unroll
  for (int i = 0; i < NQ; ++i) {
    float4 h, l;
    h.x = tf32_trunc(v[i].x); h.y = tf32_trunc(v[i].y); h.z = tf32_trunc(v[i].z); h.w = tf32_trunc(v[i].w);
    l.x = tf32_trunc(v[i].x - h.x); l.y = tf32_trunc(v[i].y - h.y);
    l.z = tf32_trunc(v[i].z - h.z); l.w = tf32_trunc(v[i].w - h.w);
    lo[t + 256 * i] = l;
    if (!RAW_HI) x[t + 256 * i] = h;
  }
}

template <int BN, bool A_MN, bool B_MN, bool RAW_HI>
__global__ void __launch_bounds__(kThreads, 1)
gemm_tma_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                const __grid_constant__ CUtensorMap tmC, TParams p) {
  using C = TCfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  uint64_t* tma_full = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES);
  uint64_t* conv_full = tma_full + C::STAGES;
  uint64_t* empty = conv_full + C::STAGES;
  uint64_t* done = empty + C::STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(done + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * BN, m0 = blockIdx.y * BM, z = blockIdx.z;
  const int nkb_total = (p.K + BK - 1) / BK;
  const int kb_begin = z * p.kb_per_split;
  const int nkb = max(0, min(nkb_total, kb_begin + p.kb_per_split) - kb_begin);

  if (threadIdx.x == 0) {
    for (int s = 0; s < C::STAGES; ++s) {
      sfdev::mbar_init(&tma_full[s], 1);
      sfdev::mbar_init(&conv_full[s], kConvWarps);
      sfdev::mbar_init(&empty[s], 1);
    }
    sfdev::mbar_init(done, 1);
    sfdev::mbar_fence_init();
    asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmA)) : "memory");
    asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmB)) : "memory");
    asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmC)) : "memory");
  }
  if (warp == kMmaWarp) sfdev::tmem_alloc<C::TMEM_COLS>(tmem_slot);
  sfdev::tc_fence_before();
  __syncthreads();
  sfdev::tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      for (int i = 0; i < nkb; ++i) {
        const int s = i % C::STAGES, round = i / C::STAGES;
        if (round > 0) sfdev::mbar_wait(&empty[s], (round - 1) & 1);
        const uint32_t st = sfdev::smem_u32(smem + s * C::STAGE_BYTES);
        const uint32_t bar = sfdev::smem_u32(&tma_full[s]);
        expect_tx(&tma_full[s], C::A_BYTES + C::B_BYTES);
        const int k0 = (kb_begin + i) * BK;
        if constexpr (A_MN) {
#pragma unroll
          for (int b = 0; b < BM / 32; ++b) tma_load_2d(st + b * 4096, &tmA, bar, m0 + 32 * b, k0);
        } else {
          tma_load_2d(st, &tmA, bar, k0, m0);
        }
        const uint32_t sb = st + 2 * C::A_BYTES;
        if constexpr (B_MN) {
#pragma unroll
          for (int b = 0; b < BN / 32; ++b) tma_load_2d(sb + b * 4096, &tmB, bar, n0 + 32 * b, k0);
        } else {
          tma_load_2d(sb, &tmB, bar, k0, n0);
        }
      }
    }
  } else if (warp <= kConvWarps) {
    const int t = threadIdx.x - 32;  // 0..255
    for (int i = 0; i < nkb; ++i) {
      const int s = i % C::STAGES;
      sfdev::mbar_wait(&tma_full[s], (i / C::STAGES) & 1);
      uint8_t* st = smem + s * C::STAGE_BYTES;
      float4* a = reinterpret_cast<float4*>(st);
      float4* alo = reinterpret_cast<float4*>(st + C::A_BYTES);
      float4* b = reinterpret_cast<float4*>(st + 2 * C::A_BYTES);
      float4* blo = reinterpret_cast<float4*>(st + 2 * C::A_BYTES + C::B_BYTES);
      split_tile<C::A_BYTES / 16 / 256, RAW_HI>(a, alo, t);
      split_tile<C::B_BYTES / 16 / 256, RAW_HI>(b, blo, t);
      sfdev::fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) sfdev::mbar_arrive(&conv_full[s]);
    }
  } else {
    // MMA issuer
    constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((A_MN ? 1u : 0u) << 15) |
                               ((B_MN ? 1u : 0u) << 16) | (uint32_t(BN >> 3) << 17) |
                               (uint32_t(BM >> 4) << 24);
    for (int i = 0; i < nkb; ++i) {
      const int s = i % C::STAGES;
      sfdev::mbar_wait(&conv_full[s], (i / C::STAGES) & 1);
      sfdev::tc_fence_after();
      if (lane == 0) {
        const uint32_t base = sfdev::smem_u32(smem + s * C::STAGE_BYTES);
        const uint32_t a_hi = base, a_lo = base + C::A_BYTES;
        const uint32_t b_hi = base + 2 * C::A_BYTES, b_lo = b_hi + C::B_BYTES;
#pragma unroll
        for (int kk = 0; kk < BK / 8; ++kk) {
          const uint32_t ao = A_MN ? kk * 1024 : kk * 32;
          const uint32_t bo = B_MN ? kk * 1024 : kk * 32;
          auto da = [&](uint32_t x) { return A_MN ? desc_mn(x + ao) : desc_k(x + ao); };
          auto db = [&](uint32_t x) { return B_MN ? desc_mn(x + bo) : desc_k(x + bo); };
          sfdev::mma_tf32(tmem, da(a_lo), db(b_hi), idesc, (i | kk) != 0);
          sfdev::mma_tf32(tmem, da(a_hi), db(b_lo), idesc, 1u);
          sfdev::mma_tf32(tmem, da(a_hi), db(b_hi), idesc, 1u);
        }
        sfdev::mma_commit(&empty[s]);
      }
      __syncwarp();
    }
    if (lane == 0) sfdev::mma_commit(done);
    __syncwarp();
  }

  if (warp >= 1 && warp <= 4) {
    sfdev::mbar_wait(done, 0);
    sfdev::tc_fence_after();
    const int q = warp & 3;  // TMEM lane quarter this warp may access
    const int row0 = q * 32;
    uint8_t* ebuf = smem + q * 2 * 4096;  // stage memory is free once `done` fired
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 32) {
      uint32_t r[32];
      sfdev::tmem_ld32(tmem + (static_cast<uint32_t>(row0) << 16) + c0, r);
      sfdev::tmem_ld_wait();
      if (nkb == 0) {
#pragma unroll
        for (int j = 0; j < 32; ++j) r[j] = 0u;
      }
      if (p.splits == 1 && p.acc) {
        const int row = m0 + row0 + lane;
        if (row < p.M)
#pragma unroll
          for (int j = 0; j < 32; ++j)
            if (n0 + c0 + j < p.N)
              r[j] = __float_as_uint(__uint_as_float(r[j]) + p.C[static_cast<size_t>(row) * p.ldc + n0 + c0 + j]);
      }
      if (p.dbg & 1) {  // debug: plain global stores of the accumulator
        const int row = m0 + row0 + lane;
        if (row < p.M && p.splits == 1)
          for (int j = 0; j < 32; ++j)
            if (n0 + c0 + j < p.N) p.C[static_cast<size_t>(row) * p.ldc + n0 + c0 + j] = __uint_as_float(r[j]);
        continue;
      }
      uint8_t* buf = ebuf + ((c0 >> 5) & 1) * 4096;
      if (c0 >= 64) {
        if (lane == 0) bulk_wait_read1();
        __syncwarp();
      }
#pragma unroll
      for (int ch = 0; ch < 8; ++ch) {
        const uint32_t off = lane * 128 + ((ch ^ (lane & 7)) << 4);
        *reinterpret_cast<uint4*>(buf + off) = make_uint4(r[4 * ch], r[4 * ch + 1], r[4 * ch + 2], r[4 * ch + 3]);
      }
      sfdev::fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) {
        if (p.splits == 1) tma_store_2d(&tmC, sfdev::smem_u32(buf), n0 + c0, m0 + row0);
        else tma_store_3d(&tmC, sfdev::smem_u32(buf), n0 + c0, m0 + row0, z);
        bulk_commit();
      }
    }
    if (lane == 0) {
      bulk_wait_all();
      asm volatile("fence.proxy.async.global;" ::: "memory");  // TMA writes before generic ops
    }
    __syncwarp();
  }
  sfdev::tc_fence_before();
  __syncthreads();
  sfdev::tc_fence_after();
  if (warp == kMmaWarp) sfdev::tmem_dealloc<C::TMEM_COLS>(tmem);
}

// Deterministic split-K reduction: C[m][n] (+)= sum_{z} ws[z][m][n].  Block = 32 float4
// output groups x 8 split lanes; lane zl sums z = zl, zl+8, ... (two accumulators), the 8
// lane partials are then combined in index order — parallel over outputs AND splits.
__global__ void __launch_bounds__(256)
splitk_reduce_kernel(const float* __restrict__ ws, float* __restrict__ C, int M, int N, int S, int ldc,
                     int acc) {
  const int lane = threadIdx.x & 31, zl = threadIdx.x >> 5;
  const uint64_t total4 = static_cast<uint64_t>(M) * N / 4;  // N % 4 == 0
  const uint64_t q = static_cast<uint64_t>(blockIdx.x) * 32 + lane;
  const size_t plane = static_cast<size_t>(M) * N;
  float4 s0 = make_float4(0.f, 0.f, 0.f, 0.f), s1 = s0;
  if (q < total4) {
    int z = zl;
    for (; z + 8 < S; z += 16) {
      const float4 a = __ldcs(reinterpret_cast<const float4*>(ws + z * plane) + q);
      const float4 b = __ldcs(reinterpret_cast<const float4*>(ws + (z + 8) * plane) + q);
      s0.x += a.x; s0.y += a.y; s0.z += a.z; s0.w += a.w;
      s1.x += b.x; s1.y += b.y; s1.z += b.z; s1.w += b.w;
    }
    if (z < S) {
      const float4 a = __ldcs(reinterpret_cast<const float4*>(ws + z * plane) + q);
      s0.x += a.x; s0.y += a.y; s0.z += a.z; s0.w += a.w;
    }
  }
  __shared__ float4 red[8][32];
  red[zl][lane] = make_float4(s0.x + s1.x, s0.y + s1.y, s0.z + s1.z, s0.w + s1.w);
  __syncthreads();
  if (zl != 0 || q >= total4) return;
  float4 t = red[0][lane];
#pragma unroll
  for (int j = 1; j < 8; ++j) {
    const float4 v = red[j][lane];
    t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
  }
  const uint64_t e = q * 4;
  const int m = static_cast<int>(e / N), n = static_cast<int>(e % N);
  float4* o = reinterpret_cast<float4*>(C + static_cast<size_t>(m) * ldc + n);
  if (acc) {
    const float4 c = *o;
    t.x = c.x + t.x; t.y = c.y + t.y; t.z = c.z + t.z; t.w = c.w + t.w;
  }
  *o = t;
}

// ---- host: tensor maps ------------------------------------------------------------------
PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  return fn;
}

bool map2d(CUtensorMap* m, const void* base, uint64_t cols, uint64_t rows, uint64_t pitch_bytes,
           uint32_t box_cols, uint32_t box_rows,
           CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  auto fn = encode_fn();
  if (!fn) return false;
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {pitch_bytes};
  cuuint32_t box[2] = {box_cols, box_rows};
  cuuint32_t es[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<void*>(base), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool map3d_ws(CUtensorMap* m, const void* base, uint64_t N, uint64_t M, uint64_t S) {
  auto fn = encode_fn();
  if (!fn) return false;
  cuuint64_t dims[3] = {N, M, S};
  cuuint64_t strides[2] = {N * 4, N * M * 4};
  cuuint32_t box[3] = {32, 32, 1};
  cuuint32_t es[3] = {1, 1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<void*>(base), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <int BN, bool AM, bool BMn, bool RAW>
cudaError_t launch_tma_t(const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& c,
                         const TParams& p, dim3 grid, cudaStream_t st) {
  auto kern = gemm_tma_kernel<BN, AM, BMn, RAW>;
  static std::atomic<uint64_t> configured{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (!(configured.load() & bit)) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, TCfg<BN>::SMEM);
    if (e != cudaSuccess) return e;
    configured.fetch_or(bit);
  }
  kern<<<grid, kThreads, TCfg<BN>::SMEM, st>>>(a, b, c, p);
  count_launch();
  return cudaGetLastError();
}

template <int BN, bool RAW>
cudaError_t dispatch_major(bool a_mn, bool b_mn, const CUtensorMap& a, const CUtensorMap& b,
                           const CUtensorMap& c, const TParams& p, dim3 grid, cudaStream_t st) {
  if (a_mn && b_mn) return launch_tma_t<BN, true, true, RAW>(a, b, c, p, grid, st);
  if (a_mn) return launch_tma_t<BN, true, false, RAW>(a, b, c, p, grid, st);
  if (b_mn) return launch_tma_t<BN, false, true, RAW>(a, b, c, p, grid, st);
  return launch_tma_t<BN, false, false, RAW>(a, b, c, p, grid, st);
}

}  // namespace

bool gemm_tma_eligible(const GemmArgs& a, int splits) {
  auto al = [](const void* p) { return reinterpret_cast<uintptr_t>(p) % 16 == 0; };
  if (!encode_fn()) return false;
  if (a.lda % 4 || a.ldb % 4 || a.ldc % 4 || !al(a.A) || !al(a.B) || !al(a.C)) return false;
  if (splits > 1 && a.N % 4) return false;
  return true;
}

cudaError_t launch_gemm_tma(const GemmArgs& a, int bn, int splits, int kb_per_split, int tiles_n,
                            int tiles_m, bool raw_hi, cudaStream_t st) {
  const bool a_mn = a.ta, b_mn = !a.tb;
  CUtensorMap ma, mb, mc;
  // A: op(A) is M x K.  Stored [M][K] (K-major) or [K][M] (MN-major).
  constexpr CUtensorMapSwizzle kMN = CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B;
  bool ok = a_mn ? map2d(&ma, a.A, a.M, a.K, static_cast<uint64_t>(a.lda) * 4, 32, 32, kMN)
                 : map2d(&ma, a.A, a.K, a.M, static_cast<uint64_t>(a.lda) * 4, 32, BM);
  // B: op(B) is K x N.  Stored [K][N] (MN-major) or [N][K] (TB, K-major).
  ok = ok && (b_mn ? map2d(&mb, a.B, a.N, a.K, static_cast<uint64_t>(a.ldb) * 4, 32, 32, kMN)
                   : map2d(&mb, a.B, a.K, a.N, static_cast<uint64_t>(a.ldb) * 4, 32, bn));
  ok = ok && (splits == 1 ? map2d(&mc, a.C, a.N, a.M, static_cast<uint64_t>(a.ldc) * 4, 32, 32)
                          : map3d_ws(&mc, a.ws, a.N, a.M, splits));
  if (!ok) return cudaErrorInvalidValue;
  static const int dbg = std::getenv("SF_GEMM_DEBUG") ? std::atoi(std::getenv("SF_GEMM_DEBUG")) : 0;
  TParams p{a.M, a.N, a.K, a.ldc, splits, kb_per_split, a.acc ? 1 : 0, dbg, a.C, a.ws, a.counters};
  dim3 grid(tiles_n, tiles_m, splits);
  cudaError_t e;
  if (bn == 64)
    e = raw_hi ? dispatch_major<64, true>(a_mn, b_mn, ma, mb, mc, p, grid, st)
               : dispatch_major<64, false>(a_mn, b_mn, ma, mb, mc, p, grid, st);
  else
    e = raw_hi ? dispatch_major<128, true>(a_mn, b_mn, ma, mb, mc, p, grid, st)
               : dispatch_major<128, false>(a_mn, b_mn, ma, mb, mc, p, grid, st);
  if (e != cudaSuccess || splits == 1) return e;
  if (a.ldc % 4 || reinterpret_cast<uintptr_t>(a.C) % 16) return cudaErrorInvalidValue;
  const uint64_t total4 = static_cast<uint64_t>(a.M) * a.N / 4;
  splitk_reduce_kernel<<<static_cast<unsigned>((total4 + 31) / 32), 256, 0, st>>>(
      a.ws, a.C, a.M, a.N, splits, a.ldc, a.acc ? 1 : 0);
  count_launch();
  return cudaGetLastError();
}

}  // namespace sfk
