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
#include <cooperative_groups.h>
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <atomic>
#include <map>
#include <mutex>
#include <tuple>

#include "sf_device.cuh"
#include "sf_kernels.h"
#include "sf_launch.cuh"

namespace sfk {
namespace {

constexpr int BM = 128;
constexpr int BK = 32;
constexpr int kConvWarps = 8;
constexpr int kMmaWarp = 9;
constexpr int kThreads = 10 * 32;

// BKT = 16 (128x256 tiles): half-depth stages, twice as many in the same shared memory, K-major
// operands in SWIZZLE_64B (64-B rows) and MN-major blocks of 32 x 16 (2 KiB)
//
// ATM (A in TMEM): the converters read the raw A tile once from shared memory and write its tf32
// hi / lo split straight into TMEM columns (tcgen05.st); the MMAs take A from TMEM and only B
// from shared memory.  Shared-memory traffic per k-block is what bounds this loop (TMA writes +
// converter reads / writes + MMA operand reads at ~128 B/clk: 192 KB -> 1500 cycles per 128x128
// k-block with A in smem, 128 KB with A in TMEM); the stage then holds A raw + B raw + B lo.
template <int BN, int BKT = BK, bool ATM = false>
struct TCfg {
  static constexpr int A_BYTES = BM * BKT * 4;
  static constexpr int B_BYTES = BN * BKT * 4;
  static constexpr int STAGE_BYTES = ATM ? A_BYTES + 2 * B_BYTES : 2 * A_BYTES + 2 * B_BYTES;
  static constexpr int STAGES = ATM ? (BN == 64 ? 6 : BN == 128 ? 4 : BKT == 16 ? 5 : 2)
                                    : BKT == 16 ? 4 : BN == 64 ? 4 : BN == 128 ? 3 : 2;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 256;
  static constexpr uint32_t TMEM_COLS = BN;
};

struct TParams {
  int M, N, K, ldc;
  int splits, kb_per_split, acc, dbg, stages;
  int cluster_reduce;  // 1: the splits of a tile form one cluster (1, 1, splits) and reduce over DSMEM
  int merge;           // 128x64 / 128x128 tiles with A in TMEM: merged A_hi.[B_hi | B_lo] MMA (MERGE)
  float* C;
  float* ws;
  unsigned* counters;
};

template <int BKT = BK>
__device__ __forceinline__ uint64_t desc_k(uint32_t saddr) {
  // K-major: BKT = 32 -> SWIZZLE_128B (layout 2, 8-row groups 1024 B apart); BKT = 16 ->
  // SWIZZLE_64B (layout 4, 8-row groups 512 B apart)
  if constexpr (BKT == 16)
    return static_cast<uint64_t>((saddr & 0x3FFFFu) >> 4) | (1ull << 16) | (32ull << 32) | (1ull << 46) |
           (4ull << 61);
  return static_cast<uint64_t>((saddr & 0x3FFFFu) >> 4) | (1ull << 16) | (64ull << 32) | (1ull << 46) |
         (2ull << 61);
}
template <int BKT = BK>
__device__ __forceinline__ uint64_t desc_mn(uint32_t saddr) {
  // MN-major 32-bit operands use SWIZZLE_128B_BASE32B (layout type 1; 32-B swizzle atoms,
  // CUTLASS Layout_MN_SW128_32B_Atom): 4-row K groups 512 B apart (SBO), 32-element MN
  // blocks 4096 B apart (LBO).  TMA writes it with CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B.
  // (BKT = 16: the MN blocks are 2048 B apart)
  return static_cast<uint64_t>((saddr & 0x3FFFFu) >> 4) | (static_cast<uint64_t>(BKT * 8) << 16) |
         (32ull << 32) | (1ull << 46) | (1ull << 61);
}

using sfdev::tma_load_2d;
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
using sfdev::expect_tx;

__device__ __forceinline__ float tf32_trunc(float x) {
  return __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
}

__device__ __forceinline__ float4 lds128(uint32_t a) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts128(uint32_t a, float4 v) {
  asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" :: "r"(a), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
}

// Split NQ float4 of a tile (thread stride 256): lo = tf32(x - trunc_tf32(x)) into `lo`;
// unless RAW_HI, also overwrite x with trunc_tf32(x).  All loads are issued first; explicit
// shared-space accesses (LDS/STS.128, not generic LD/ST).
template <int NQ, bool RAW_HI>
__device__ __forceinline__ void split_tile(float4* __restrict__ x, float4* __restrict__ lo, int t) {
  const uint32_t xs = sfdev::smem_u32(x) + 16u * t, ls = sfdev::smem_u32(lo) + 16u * t;
  float4 v[NQ];
#pragma unroll
  for (int i = 0; i < NQ; ++i) v[i] = lds128(xs + 4096u * i);
#pragma unroll
  for (int i = 0; i < NQ; ++i) {
    float4 h, l;
    h.x = tf32_trunc(v[i].x); h.y = tf32_trunc(v[i].y); h.z = tf32_trunc(v[i].z); h.w = tf32_trunc(v[i].w);
    l.x = tf32_trunc(v[i].x - h.x); l.y = tf32_trunc(v[i].y - h.y);
    l.z = tf32_trunc(v[i].z - h.z); l.w = tf32_trunc(v[i].w - h.w);
    sts128(ls + 4096u * i, l);
    if (!RAW_HI) sts128(xs + 4096u * i, h);
  }
}

__device__ __forceinline__ float lds32(uint32_t a) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
  return v;
}
template <int NR>
__device__ __forceinline__ void tmem_st(uint32_t taddr, const float (&v)[NR]) {  // 32x32b.xNR
  static_assert(NR == 8 || NR == 16, "tmem_st: 8 or 16 columns");
  if constexpr (NR == 16)
    asm volatile("tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};"
                 :: "r"(taddr), "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]),
                    "f"(v[7]), "f"(v[8]), "f"(v[9]), "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]),
                    "f"(v[15]) : "memory");
  else
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
                 :: "r"(taddr), "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]),
                    "f"(v[7]) : "memory");
}
__device__ __forceinline__ void mma_tf32_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                            uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}"
      :: "r"(d_tmem), "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate));
}

// Split-K reduction of one tile over its cluster (S CTAs, rank = split index z): CTA z sums its
// 1/S share of the tile's 16-B chunks over the S partials (32x32 swizzled blocks in each CTA's
// smem) in the fixed order 0..S-1, then + C when accumulating.  Loads go out in batches of
// about 16 remote 16-B reads per thread before any is consumed (one DSMEM round trip per batch).
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t cluster_map(uint32_t saddr, int rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}

// Split-K reduction of one tile inside its cluster (S CTAs, rank = split z).  Every CTA holds
// its fp32 partial in smem [0, T) as 32x32 swizzled blocks (block = col block * 4 + quarter).
// Owner z reduces the 16-B chunks [z PER, (z+1) PER): each other CTA pushes that range of its
// partial into the owner's receive slot with ONE bulk DSMEM copy (completion on the owner's
// mbarrier), then the owner sums its own and the S-1 received ranges from local smem in the
// fixed order z' = 0..S-1 (+ C when accumulating) and stores the chunks to C.
template <int BN>
__device__ __forceinline__ void cluster_push_reduce(uint8_t* smem, uint64_t* red_bar, const TParams& p, int m0,
                                                    int n0, int z) {
  constexpr int T = BM * BN * 4, TOT = T / 16;
  const int S = p.splits;
  const int PER = (TOT + S - 1) / S;
  auto len = [&](int o) { return max(0, min(TOT, (o + 1) * PER) - o * PER); };
  const uint32_t sbase = sfdev::smem_u32(smem), bar = sfdev::smem_u32(red_bar);
  if (threadIdx.x == 0) {
    const int mine = len(z);
    if (mine > 0) expect_tx(red_bar, static_cast<uint32_t>((S - 1) * mine * 16));
    else sfdev::mbar_arrive(red_bar);
    for (int o = 0; o < S; ++o) {
      if (o == z || len(o) == 0) continue;
      const int slot = z < o ? z : z - 1;
      const uint32_t dst = cluster_map(sbase + T + slot * PER * 16, o);
      asm volatile("cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   :: "r"(dst), "r"(sbase + o * PER * 16), "r"(len(o) * 16), "r"(cluster_map(bar, o)) : "memory");
    }
  }
  sfdev::mbar_wait(red_bar, 0);
  const int c_beg = z * PER, c_end = c_beg + len(z);
  for (int c = c_beg + static_cast<int>(threadIdx.x); c < c_end; c += kThreads) {
    const int off = c * 16;
    const int block = off >> 12, within = off & 4095;
    const int ln = within >> 7, ch = ((within >> 4) & 7) ^ (ln & 7);
    const int row = (block & 3) * 32 + ln, col4 = (block >> 2) * 8 + ch;
    const int gr = m0 + row, gc = n0 + col4 * 4;
    float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int zz = 0; zz < S; ++zz) {
      const uint32_t a = zz == z ? sbase + off : sbase + T + (zz < z ? zz : zz - 1) * PER * 16 + (c - c_beg) * 16;
      const float4 v = lds128(a);
      if (zz == 0) t = v;
      else { t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w; }
    }
    if (gr >= p.M || gc >= p.N) continue;
    float4* o = reinterpret_cast<float4*>(p.C + static_cast<size_t>(gr) * p.ldc + gc);
    if (p.acc) {
      const float4 cv = *o;
      t.x = cv.x + t.x; t.y = cv.y + t.y; t.z = cv.z + t.z; t.w = cv.w + t.w;
    }
    *o = t;
  }
}

// 128x64 tiles run two CTAs per SM when the grid has more tiles than SMs (2-stage ring): the
// register budget must leave room for both (<= 96 per thread at 320 threads)
template <int BN, bool A_MN, bool B_MN, bool RAW_HI, int BKT = BK, bool ATM = false>
__global__ void __launch_bounds__(kThreads, BN == 64 ? 2 : 1)
gemm_tma_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                const __grid_constant__ CUtensorMap tmC, TParams p) {
  using C = TCfg<BN, BKT, ATM>;
  constexpr int BK = BKT;  // k-block depth of this instantiation
  // MERGE (128x64 / 128x128 tiles, A in TMEM): A_hi.B_hi and A_hi.B_lo in ONE N=2BN MMA over
  // the adjacent B_hi | B_lo stage buffers into two BN-column accumulators (+ A_lo.B_hi into
  // the first), summed in the epilogue: 2 MMAs per K step instead of 3 (an MMA instruction
  // costs more than its N x 8 x 128 share of the tensor pipe in this loop)
  const bool MERGE = ATM && BN <= 128 && p.merge;
  const int ACC = MERGE ? 2 * BN : BN;  // accumulator TMEM columns
  const int NS = p.stages;  // ring depth (<= C::STAGES; 2 for short K: two CTAs per SM)
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  uint64_t* tma_full = reinterpret_cast<uint64_t*>(smem + NS * C::STAGE_BYTES);
  uint64_t* conv_full = tma_full + NS;
  uint64_t* empty = conv_full + NS;
  uint64_t* done = empty + NS;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(done + 1);
  uint64_t* red_bar = done + 2;  // split-K cluster reduction (receive slots complete here)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * BN, m0 = blockIdx.y * BM, z = blockIdx.z;
  __shared__ long long tsd[8];  // phase probe (SF_GEMM_DEBUG bit 3: clock64 stamps, printf of 3 CTAs)
  if ((p.dbg & 8) && threadIdx.x == 0) tsd[0] = clock64();
  const int nkb_total = (p.K + BK - 1) / BK;
  const int kb_begin = z * p.kb_per_split;
  const int nkb = max(0, min(nkb_total, kb_begin + p.kb_per_split) - kb_begin);
  if (threadIdx.x == 0) {
    for (int s = 0; s < NS; ++s) {
      sfdev::mbar_init(&tma_full[s], 1);
      sfdev::mbar_init(&conv_full[s], kConvWarps);
      sfdev::mbar_init(&empty[s], 1);
    }
    sfdev::mbar_init(red_bar, 1);
    sfdev::mbar_init(done, 1);
    sfdev::mbar_fence_init();
    asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmA)) : "memory");
    asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmB)) : "memory");
    asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmC)) : "memory");
  }
  // ATM: accumulator in columns [0, BN), stage s's A hi / lo at BN + 2 s BK (+ BK); a 2-stage
  // ring (two CTAs per SM) fits 256 columns, deeper rings take all 512
  const bool tm_small = !ATM || ACC + NS * 2 * BK <= 256;
  if (warp == kMmaWarp) {
    if (!ATM) sfdev::tmem_alloc<C::TMEM_COLS>(tmem_slot);
    else if (tm_small) sfdev::tmem_alloc<256>(tmem_slot);
    else sfdev::tmem_alloc<512>(tmem_slot);
  }
  sfdev::tc_fence_before();
  __syncthreads();
  sfdev::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  if ((p.dbg & 8) && threadIdx.x == 0) tsd[1] = clock64();

  if (warp == 0) {
    if (lane == 0) {
      for (int i = 0; i < nkb; ++i) {
        const int s = i % NS, round = i / NS;
        if (round > 0) sfdev::mbar_wait(&empty[s], (round - 1) & 1);
        const uint32_t st = sfdev::smem_u32(smem + s * C::STAGE_BYTES);
        const uint32_t bar = sfdev::smem_u32(&tma_full[s]);
        expect_tx(&tma_full[s], C::A_BYTES + C::B_BYTES);
        const int k0 = (kb_begin + i) * BK;
        if constexpr (A_MN) {
#pragma unroll
          for (int b = 0; b < BM / 32; ++b) tma_load_2d(st + b * (BK * 128), &tmA, bar, m0 + 32 * b, k0);
        } else {
          tma_load_2d(st, &tmA, bar, k0, m0);
        }
        const uint32_t sb = st + (ATM ? 1 : 2) * C::A_BYTES;
        if constexpr (B_MN) {
#pragma unroll
          for (int b = 0; b < BN / 32; ++b) tma_load_2d(sb + b * (BK * 128), &tmB, bar, n0 + 32 * b, k0);
        } else {
          tma_load_2d(sb, &tmB, bar, k0, n0);
        }
      }
    }
  } else if (ATM && warp <= kConvWarps) {
    // B: lo split in shared memory (all 256 threads).  A: warp w owns TMEM lane quarter w % 4
    // (rows 32 q + lane) and K half h; its thread reads its row's BK / 2 raw values, writes
    // hi = raw (the MMA reads only the tf32 bits) and lo = tf32(x - tf32(x)) into TMEM.
    const int t = threadIdx.x - 32;
    const int q = warp & 3, h = (warp - 1) >> 2;
    constexpr int KH = BK / 2;
    const int r = 32 * q + lane;
    const uint32_t lane_base = static_cast<uint32_t>(32 * q) << 16;
    for (int i = 0; i < nkb; ++i) {
      const int s = i % NS;
      sfdev::mbar_wait(&tma_full[s], (i / NS) & 1);
      if ((p.dbg & 8) && i == 0 && threadIdx.x == 32) tsd[2] = clock64();
      uint8_t* st = smem + s * C::STAGE_BYTES;
      const uint32_t sa = sfdev::smem_u32(st);
      float x[KH];
      if constexpr (A_MN) {  // SWIZZLE_128B rows of 32 M (one block per quarter), BK rows of K
        const uint32_t base = sa + q * (BK * 128) + (lane & 3) * 4;
#pragma unroll
        for (int j = 0; j < KH; ++j) {
          const int k = h * KH + j;
          x[j] = lds32(base + k * 128 + ((((lane >> 2) ^ (k & 7))) << 4));
        }
      } else if constexpr (BK == 32) {  // K-major SWIZZLE_128B: 128-B rows
#pragma unroll
        for (int cc = 0; cc < KH / 4; ++cc) {
          const int c = h * (KH / 4) + cc;
          const float4 v = lds128(sa + r * 128 + ((c ^ (r & 7)) << 4));
          x[4 * cc] = v.x; x[4 * cc + 1] = v.y; x[4 * cc + 2] = v.z; x[4 * cc + 3] = v.w;
        }
      } else {  // K-major SWIZZLE_64B: 64-B rows
#pragma unroll
        for (int cc = 0; cc < KH / 4; ++cc) {
          const int c = h * (KH / 4) + cc;
          const float4 v = lds128(sa + r * 64 + ((c ^ ((r >> 1) & 3)) << 4));
          x[4 * cc] = v.x; x[4 * cc + 1] = v.y; x[4 * cc + 2] = v.z; x[4 * cc + 3] = v.w;
        }
      }
      if (!(p.dbg & 2)) {
        float lo[KH];
#pragma unroll
        for (int j = 0; j < KH; ++j) lo[j] = tf32_trunc(x[j] - tf32_trunc(x[j]));
        const uint32_t col = static_cast<uint32_t>(ACC + s * 2 * BK + h * KH);
        tmem_st<KH>(tmem + lane_base + col, x);
        tmem_st<KH>(tmem + lane_base + col + BK, lo);
        float4* b = reinterpret_cast<float4*>(st + C::A_BYTES);
        float4* blo = reinterpret_cast<float4*>(st + C::A_BYTES + C::B_BYTES);
        split_tile<C::B_BYTES / 16 / 256, true>(b, blo, t);
      } else {
        tmem_st<KH>(tmem + lane_base + static_cast<uint32_t>(ACC + s * 2 * BK + h * KH), x);
      }
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      sfdev::fence_proxy_async_smem();
      sfdev::tc_fence_before();
      __syncwarp();
      if (lane == 0) sfdev::mbar_arrive(&conv_full[s]);
    }
  } else if (warp <= kConvWarps) {
    const int t = threadIdx.x - 32;  // 0..255
    for (int i = 0; i < nkb; ++i) {
      const int s = i % NS;
      sfdev::mbar_wait(&tma_full[s], (i / NS) & 1);
      if ((p.dbg & 8) && i == 0 && threadIdx.x == 32) tsd[2] = clock64();
      uint8_t* st = smem + s * C::STAGE_BYTES;
      float4* a = reinterpret_cast<float4*>(st);
      float4* alo = reinterpret_cast<float4*>(st + C::A_BYTES);
      float4* b = reinterpret_cast<float4*>(st + 2 * C::A_BYTES);
      float4* blo = reinterpret_cast<float4*>(st + 2 * C::A_BYTES + C::B_BYTES);
      if (!(p.dbg & 2)) {  // dbg bit 1 (probe only, wrong results): skip the split
        split_tile<C::A_BYTES / 16 / 256, RAW_HI>(a, alo, t);
        split_tile<C::B_BYTES / 16 / 256, RAW_HI>(b, blo, t);
      }
      sfdev::fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) sfdev::mbar_arrive(&conv_full[s]);
    }
  } else {
    // MMA issuer
    constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((A_MN && !ATM ? 1u : 0u) << 15) |
                               ((B_MN ? 1u : 0u) << 16) | (uint32_t(BN >> 3) << 17) |
                               (uint32_t(BM >> 4) << 24);
    for (int i = 0; i < nkb; ++i) {
      const int s = i % NS;
      sfdev::mbar_wait(&conv_full[s], (i / NS) & 1);
      sfdev::tc_fence_after();
      if (ATM && lane == 0) {
        const uint32_t b_hi = sfdev::smem_u32(smem + s * C::STAGE_BYTES) + C::A_BYTES, b_lo = b_hi + C::B_BYTES;
        const uint32_t a_hi = tmem + static_cast<uint32_t>(ACC + s * 2 * BK), a_lo = a_hi + BK;
#pragma unroll
        for (int kk = 0; kk < BK / 8; ++kk) {
          const uint32_t bo = B_MN ? kk * 1024 : kk * 32;
          auto db = [&](uint32_t x) { return B_MN ? desc_mn<BK>(x + bo) : desc_k<BK>(x + bo); };
          if (MERGE) {
            constexpr uint32_t idesc2 = (idesc & ~(0x3Fu << 17)) | (uint32_t((2 * BN) >> 3) << 17);
            mma_tf32_ts(tmem, a_hi + kk * 8, db(b_hi), idesc2, (i | kk) != 0);  // [B_hi | B_lo]
            mma_tf32_ts(tmem, a_lo + kk * 8, db(b_hi), idesc, 1u);
            continue;
          }
          if (!(p.dbg & 4)) {
            mma_tf32_ts(tmem, a_lo + kk * 8, db(b_hi), idesc, (i | kk) != 0);
            mma_tf32_ts(tmem, a_hi + kk * 8, db(b_lo), idesc, 1u);
          }
          mma_tf32_ts(tmem, a_hi + kk * 8, db(b_hi), idesc, (p.dbg & 4) ? ((i | kk) != 0) : 1u);
        }
        sfdev::mma_commit(&empty[s]);
      } else if (!ATM && lane == 0) {
        const uint32_t base = sfdev::smem_u32(smem + s * C::STAGE_BYTES);
        const uint32_t a_hi = base, a_lo = base + C::A_BYTES;
        const uint32_t b_hi = base + 2 * C::A_BYTES, b_lo = b_hi + C::B_BYTES;
#pragma unroll
        for (int kk = 0; kk < BK / 8; ++kk) {
          const uint32_t ao = A_MN ? kk * 1024 : kk * 32;
          const uint32_t bo = B_MN ? kk * 1024 : kk * 32;
          auto da = [&](uint32_t x) { return A_MN ? desc_mn<BK>(x + ao) : desc_k<BK>(x + ao); };
          auto db = [&](uint32_t x) { return B_MN ? desc_mn<BK>(x + bo) : desc_k<BK>(x + bo); };
          if (!(p.dbg & 4)) {  // dbg bit 2 (probe only, wrong results): hi.hi MMA alone
            sfdev::mma_tf32(tmem, da(a_lo), db(b_hi), idesc, (i | kk) != 0);
            sfdev::mma_tf32(tmem, da(a_hi), db(b_lo), idesc, 1u);
          }
          sfdev::mma_tf32(tmem, da(a_hi), db(b_hi), idesc, (p.dbg & 4) ? ((i | kk) != 0) : 1u);
        }
        sfdev::mma_commit(&empty[s]);
      }
      __syncwarp();
    }
    if ((p.dbg & 8) && lane == 0) tsd[3] = clock64();
    if (lane == 0) sfdev::mma_commit(done);
    __syncwarp();
  }

  if (warp >= 1 && warp <= 4) {
    sfdev::mbar_wait(done, 0);
    sfdev::tc_fence_after();
    if ((p.dbg & 8) && threadIdx.x == 32) tsd[4] = clock64();
    const int q = warp & 3;  // TMEM lane quarter this warp may access
    const int row0 = q * 32;
    uint8_t* ebuf = smem + q * 2 * 4096;  // stage memory is free once `done` fired
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 32) {
      uint32_t r[32];
      sfdev::tmem_ld32(tmem + (static_cast<uint32_t>(row0) << 16) + c0, r);
      sfdev::tmem_ld_wait();
      if (MERGE) {  // + the A_hi.B_lo half
        uint32_t r2[32];
        sfdev::tmem_ld32(tmem + (static_cast<uint32_t>(row0) << 16) + BN + c0, r2);
        sfdev::tmem_ld_wait();
#pragma unroll
        for (int j = 0; j < 32; ++j) r[j] = __float_as_uint(__uint_as_float(r[j]) + __uint_as_float(r2[j]));
      }
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
      if (p.cluster_reduce) {  // this split's partial -> own smem, 32x32 blocks (col block, quarter)
        uint8_t* blk = smem + ((c0 >> 5) * 4 + q) * 4096;
#pragma unroll
        for (int ch = 0; ch < 8; ++ch) {
          const uint32_t off = lane * 128 + ((ch ^ (lane & 7)) << 4);
          *reinterpret_cast<uint4*>(blk + off) = make_uint4(r[4 * ch], r[4 * ch + 1], r[4 * ch + 2], r[4 * ch + 3]);
        }
        sfdev::fence_proxy_async_smem();  // the partial leaves by bulk copy (async proxy)
        continue;
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
  if ((p.dbg & 8) && threadIdx.x == 32) tsd[5] = clock64();
  if (p.cluster_reduce) {
    // split-K without a workspace: the tile's S splits are one cluster (cluster_push_reduce)
    __syncwarp();
    cluster_sync_all();  // every partial in smem (made visible to the async proxy by its writers)
    if ((p.dbg & 8) && threadIdx.x == 0) tsd[6] = clock64();
    cluster_push_reduce<BN>(smem, red_bar, p, m0, n0, z);
    __syncwarp();
    cluster_sync_all();  // no CTA leaves (freeing its smem) while a peer still copies from it
  }
  sfdev::tc_fence_before();
  __syncthreads();
  sfdev::tc_fence_after();
  if ((p.dbg & 8) && threadIdx.x == 0) {
    tsd[7] = clock64();
    const unsigned bid = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
    if (bid == 0 || bid == gridDim.x * gridDim.y * gridDim.z - 1 || bid == 37)
      printf("PHASE bid %u nkb %d setup %lld firstTMA %lld mma_end %lld epi_start %lld epi_end %lld cl1 %lld end %lld\n",
             bid, nkb, tsd[1] - tsd[0], tsd[2] - tsd[0], tsd[3] - tsd[0], tsd[4] - tsd[0], tsd[5] - tsd[0],
             p.cluster_reduce ? tsd[6] - tsd[0] : -1ll, tsd[7] - tsd[0]);
  }
  if (warp == kMmaWarp) {
    if (!ATM) sfdev::tmem_dealloc<C::TMEM_COLS>(tmem);
    else if (tm_small) sfdev::tmem_dealloc<256>(tmem);
    else sfdev::tmem_dealloc<512>(tmem);
  }
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


// ---- TMA-streamed cluster GEMV (M <= 8, the inference path of SURVEY.md 8(a) C4) ----------
// y[m][n] = sum_k x[m][k] W[k][n] (+ C if acc) (+ bias...) (ReLU): HBM-bound on W.  A cluster
// of kGvCluster CTAs splits K; each CTA owns BC columns x kper rows of W.  Warp 8 (one thread)
// streams W as {BC cols x 32 rows} TMA boxes through a 64 KB mbarrier ring, so every CTA has
// 64 KB of loads in flight from its first cycle (the register-streamed kernels depended on
// ptxas keeping loads ahead of their FMAs, which it does not).  Warps 0-7: thread = (row lane
// rl, column quad qi), QW = BC/4 quads x RL = 256/QW row lanes; x is staged in smem while the
// first boxes are in flight.  Reduction: row lanes in smem in fixed order, then the cluster
// leader sums the kGvCluster partials over DSMEM in rank order (deterministic, one launch).
constexpr int kGvCluster = 8;
constexpr int kGvRows = 32;            // rows per TMA box
constexpr int kGvRing = 64 * 1024;     // bytes of W in flight per CTA
constexpr int kGvMaxKper = 1024;       // x slice staged in smem (K <= 8192)
constexpr int kGvPrefetch = 8;         // l2_hint flag: prefetch the W slice into L2 up front

template <int MR, int BC>
struct GvCfg {
  static constexpr int QW = BC / 4, RL = 256 / QW, BOX = BC * kGvRows * 4, S = kGvRing / BOX;
  static constexpr int RED = RL * QW * 16, PART = MR * QW * 16;
  static size_t smem(int kper) { return kGvRing + RED + PART + 2 * S * 8 + size_t(MR) * kper * 4 + 128; }
};

template <int MR, int BC>
__global__ void __cluster_dims__(kGvCluster, 1, 1) __launch_bounds__(288)
gemv_tma_kernel(const __grid_constant__ CUtensorMap tmW, const float* __restrict__ X,
                float* __restrict__ Y, int M, int N, int K, int ldx, int ldy, int kper, int acc,
                const float* __restrict__ b1, const float* __restrict__ b2,
                const float* __restrict__ b3, int relu, int b_const, int l2_hint,
                float* __restrict__ sm_out, int sm_ldo, unsigned* __restrict__ sm_counter,
                const char* __restrict__ pf, unsigned long long pf_bytes) {
  using Cfg = GvCfg<MR, BC>;
  constexpr int QW = Cfg::QW, RL = Cfg::RL, S = Cfg::S;
  extern __shared__ __align__(1024) unsigned char gv_smem[];
  float4* ring = reinterpret_cast<float4*>(gv_smem);
  float4* red = reinterpret_cast<float4*>(gv_smem + kGvRing);
  float4* part = reinterpret_cast<float4*>(gv_smem + kGvRing + Cfg::RED);
  uint64_t* full = reinterpret_cast<uint64_t*>(gv_smem + kGvRing + Cfg::RED + Cfg::PART);
  uint64_t* empty = full + S;
  float* xs = reinterpret_cast<float*>(empty + S);

  namespace cg = cooperative_groups;
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = static_cast<int>(cluster.block_rank());
  const int cb = blockIdx.x / kGvCluster;
  const int c0 = cb * BC;
  const int k0 = rank * kper, k1 = min(K, k0 + kper);
  const int nbox = k1 > k0 ? (k1 - k0 + kGvRows - 1) / kGvRows : 0;
  const int tid = threadIdx.x, warp = tid >> 5;

  if (tid == 0) {
    for (int i = 0; i < S; ++i) {
      sfdev::mbar_init(&full[i], 1);
      sfdev::mbar_init(&empty[i], 8);
    }
    sfdev::mbar_fence_init();
  }
  __syncthreads();

  float4 accv[MR];
#pragma unroll
  for (int m = 0; m < MR; ++m) accv[m] = make_float4(0.f, 0.f, 0.f, 0.f);
  const int qi = tid % QW, rl = tid / QW;

  sfdev::griddep_launch();  // single wave: the next layer may start its own W stream now
  if (warp == 8) {
    if ((tid & 31) == 0) {
      if (!b_const) sfdev::griddep_wait();  // W may be written by the predecessor
      const int hint = l2_hint & 3;
      const uint64_t pol = sfdev::l2_policy(hint);
      if (l2_hint & kGvPrefetch) {
        // the whole slice beyond the ring goes to L2 now: DRAM works ahead of the ring (and,
        // under PDL, while the predecessor layer drains); the ring's loads then hit L2
        for (int i = S; i < nbox; ++i) sfdev::tma_prefetch_2d(&tmW, c0, k0 + i * kGvRows);
      }
      for (int i = 0; i < nbox; ++i) {
        const int slot = i % S;
        if (i >= S) sfdev::mbar_wait(&empty[slot], ((i / S) - 1) & 1);
        expect_tx(&full[slot], Cfg::BOX);
        if (hint)  // keep (persisting set-aside) / stream (evict first) the weights
          sfdev::tma_load_2d_hint(sfdev::smem_u32(ring) + slot * Cfg::BOX, &tmW, sfdev::smem_u32(&full[slot]),
                                  c0, k0 + i * kGvRows, pol);
        else
          tma_load_2d(sfdev::smem_u32(ring) + slot * Cfg::BOX, &tmW, sfdev::smem_u32(&full[slot]), c0,
                      k0 + i * kGvRows);
      }
      // the NEXT layer's weights (constant) to L2 once this CTA's own stream is issued: HBM
      // keeps streaming through this layer's reduction, the next launch and its ramp (DESIGN.md
      // reading Q39); this CTA's share of [pf, pf + pf_bytes) in 64 KB bulk prefetches
      if (pf != nullptr && pf_bytes > 0) {
        const unsigned long long G = gridDim.x;
        const unsigned long long lo = (pf_bytes * blockIdx.x / G) & ~15ull;
        const unsigned long long hi = blockIdx.x + 1 == G ? pf_bytes : (pf_bytes * (blockIdx.x + 1) / G) & ~15ull;
        for (unsigned long long o = lo; o < hi; o += 65536) {
          const unsigned n = static_cast<unsigned>(hi - o < 65536 ? hi - o : 65536);
          asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(pf + o), "r"(n) : "memory");
        }
      }
    }
    __syncwarp();
  } else {
    sfdev::griddep_wait();  // x is the predecessor's output
    for (int i = tid; i < MR * kper; i += 256) {
      const int m = i / kper, kk = i % kper;
      xs[i] = (m < M && k0 + kk < k1) ? X[static_cast<size_t>(m) * ldx + k0 + kk] : 0.f;
    }
    asm volatile("bar.sync 1, 256;" ::: "memory");
    for (int i = 0; i < nbox; ++i) {
      const int slot = i % S;
      sfdev::mbar_wait(&full[slot], (i / S) & 1);
      const float4* tile = ring + slot * (Cfg::BOX / 16);
#pragma unroll
      for (int r = rl; r < kGvRows; r += RL) {
        const float4 w = tile[r * QW + qi];
        const int kk = i * kGvRows + r;
#pragma unroll
        for (int m = 0; m < MR; ++m) {
          const float xv = xs[m * kper + kk];
          accv[m].x = fmaf(xv, w.x, accv[m].x); accv[m].y = fmaf(xv, w.y, accv[m].y);
          accv[m].z = fmaf(xv, w.z, accv[m].z); accv[m].w = fmaf(xv, w.w, accv[m].w);
        }
      }
      __syncwarp();
      if ((tid & 31) == 0) sfdev::mbar_arrive(&empty[slot]);
    }
  }
#pragma unroll
  for (int m = 0; m < MR; ++m) {
    if (tid < 256) red[rl * QW + qi] = accv[m];
    __syncthreads();
    if (tid < QW) {
      float4 t = red[tid];
#pragma unroll 8
      for (int j = 1; j < RL; ++j) {
        const float4 v = red[j * QW + tid];
        t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
      }
      part[m * QW + tid] = t;
    }
    __syncthreads();
  }
  cluster.sync();
  if (rank == 0 && tid < MR * QW) {
    const int m = tid / QW, n = c0 + 4 * (tid % QW);
    if (m < M && n < N) {
      float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int r = 0; r < kGvCluster; ++r) {
        const float4 v = cluster.map_shared_rank(part, r)[tid];
        t.x += v.x; t.y += v.y; t.z += v.z; t.w += v.w;
      }
      float* o = Y + static_cast<size_t>(m) * ldy + n;
      const float r4[4] = {t.x, t.y, t.z, t.w};
#pragma unroll
      for (int j = 0; j < 4; ++j) {
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
    // fused row softmax: the last column block to publish its outputs normalises all rows
    // (threadfence-reduction pattern; fixed-order reductions, so results are deterministic)
    __shared__ int sm_last;
    __shared__ float sm_red[9];
    __threadfence();
    __syncthreads();
    if (tid == 0) sm_last = atomicAdd(sm_counter, 1u) == gridDim.x / kGvCluster - 1;
    __syncthreads();
    if (sm_last) {
      __threadfence();
      const int lane = tid & 31;
      for (int m = 0; m < M; ++m) {
        const float* yr = Y + static_cast<size_t>(m) * ldy;
        float mx = -INFINITY;
        for (int n = tid; n < N; n += 288) mx = fmaxf(mx, __ldcg(yr + n));
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        if (lane == 0) sm_red[warp] = mx;
        __syncthreads();
        mx = sm_red[0];
#pragma unroll
        for (int w = 1; w < 9; ++w) mx = fmaxf(mx, sm_red[w]);
        __syncthreads();
        float s = 0.f;
        for (int n = tid; n < N; n += 288) s += expf(__ldcg(yr + n) - mx);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        if (lane == 0) sm_red[warp] = s;
        __syncthreads();
        s = sm_red[0];
#pragma unroll
        for (int w = 1; w < 9; ++w) s += sm_red[w];
        __syncthreads();
        float* orow = sm_out + static_cast<size_t>(m) * sm_ldo;
        for (int n = tid; n < N; n += 288) orow[n] = expf(__ldcg(yr + n) - mx) / s;
      }
      if (tid == 0) *sm_counter = 0u;
    }
  }
  cluster.sync();
}

// ---- row-contiguous GEMV (M <= 8, B stored [N][K]: the inference weight layout) ---------
// y[m][n] = act(sum_k x[m][k] B[n][k] + biases): every output is the dot product of x with one
// contiguous row of B, so each CTA's work is ONE contiguous span of rows [r0, r1) streamed
// sequentially by 1-D bulk copies (one row per ring slot) — the DRAM access pattern of a pure
// read stream, no split-K, no cluster reduction.  Warp 8 lane 0 is the producer; ring slot s
// is always consumed by warp s % NW (NW = min(8, slots)), which takes its rows in order, so
// no consumer can run a phase ahead on a slot (lane j: float4 j, j + 32, ...; shuffle-tree
// reduce, fixed order, deterministic).  Weights that no running kernel writes (b_const) stream before
// griddep_wait(), so under PDL a layer's rows arrive while its predecessor drains; one CTA per
// SM leaves room for the next layer's CTA.  Optional fused row softmax as in gemv_tma_kernel.
constexpr int kGrRing = 96 * 1024;   // bytes of rows in flight per CTA
constexpr int kGrMaxRow = 32 * 1024;  // K <= 8192
constexpr int kGrMaxX = 64 * 1024;    // M * K * 4: x staged in smem

template <int MR>
__global__ void __launch_bounds__(288)
gemv_rows_kernel(const float* __restrict__ Bm, const float* __restrict__ X, float* __restrict__ Y,
                 int M, int N, int K, int ldb, int ldx, int ldy, int slots,
                 const float* __restrict__ b1, const float* __restrict__ b2,
                 const float* __restrict__ b3, int relu, int b_const, int l2_hint,
                 float* __restrict__ sm_out, int sm_ldo, unsigned* __restrict__ sm_counter) {
  extern __shared__ __align__(1024) unsigned char gr_smem[];
  const int rowf = K;                        // floats per row (K % 4 == 0)
  const uint32_t row_bytes = static_cast<uint32_t>(K) * 4;
  const int slot_f = (rowf + 31) / 32 * 32;  // 128-B aligned slots
  float* ring = reinterpret_cast<float*>(gr_smem);
  float* xs = ring + static_cast<size_t>(slots) * slot_f;
  uint64_t* full = reinterpret_cast<uint64_t*>(xs + static_cast<size_t>(MR) * K);
  uint64_t* empty = full + slots;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  // balanced contiguous row span of this CTA
  const int r0 = static_cast<int>(static_cast<int64_t>(N) * blockIdx.x / gridDim.x);
  const int r1 = static_cast<int>(static_cast<int64_t>(N) * (blockIdx.x + 1) / gridDim.x);
  const int nrows = r1 - r0;
  if (tid == 0) {
    for (int i = 0; i < slots; ++i) {
      sfdev::mbar_init(&full[i], 1);
      sfdev::mbar_init(&empty[i], 1);
    }
    sfdev::mbar_fence_init();
  }
  __syncthreads();
  sfdev::griddep_launch();  // the next layer may start streaming its own rows now
  if (warp == 8) {
    if (lane == 0) {
      if (!b_const) sfdev::griddep_wait();  // B may be written by the predecessor
      const uint64_t pol = sfdev::l2_policy(l2_hint);
      for (int i = 0; i < nrows; ++i) {
        const int s = i % slots;
        if (i >= slots) sfdev::mbar_wait(&empty[s], ((i / slots) - 1) & 1);
        expect_tx(&full[s], row_bytes);
        const uint32_t dst = sfdev::smem_u32(ring + static_cast<size_t>(s) * slot_f);
        const float* src = Bm + static_cast<size_t>(r0 + i) * ldb;
        if (l2_hint) sfdev::bulk_load_1d_hint(dst, src, row_bytes, sfdev::smem_u32(&full[s]), pol);
        else sfdev::bulk_load_1d(dst, src, row_bytes, sfdev::smem_u32(&full[s]));
      }
    }
    __syncwarp();
  } else {
    sfdev::griddep_wait();  // x is the predecessor's output
    for (int i = tid; i < MR * K; i += 256) {
      const int m = i / K, k = i % K;
      xs[i] = m < M ? X[static_cast<size_t>(m) * ldx + k] : 0.f;
    }
    asm volatile("bar.sync 1, 256;" ::: "memory");
    const int nq = K / 4;
    const float4* x4 = reinterpret_cast<const float4*>(xs);
    const int nw = slots < 8 ? slots : 8;
    for (int i = 0; i < nrows; ++i) {
      const int s = i % slots;
      if (s % nw != warp) continue;
      sfdev::mbar_wait(&full[s], (i / slots) & 1);
      const float4* w4 = reinterpret_cast<const float4*>(ring + static_cast<size_t>(s) * slot_f);
      float acc[MR];
#pragma unroll
      for (int m = 0; m < MR; ++m) acc[m] = 0.f;
#pragma unroll 4
      for (int q = lane; q < nq; q += 32) {
        const float4 w = w4[q];
#pragma unroll
        for (int m = 0; m < MR; ++m) {
          const float4 xv = x4[m * nq + q];
          acc[m] = fmaf(xv.x, w.x, acc[m]);
          acc[m] = fmaf(xv.y, w.y, acc[m]);
          acc[m] = fmaf(xv.z, w.z, acc[m]);
          acc[m] = fmaf(xv.w, w.w, acc[m]);
        }
      }
      __syncwarp();
      if (lane == 0) sfdev::mbar_arrive(&empty[s]);
#pragma unroll
      for (int m = 0; m < MR; ++m)
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) acc[m] += __shfl_xor_sync(0xffffffffu, acc[m], o);
      if (lane < MR && lane < M) {
        float v = 0.f;
#pragma unroll
        for (int m = 0; m < MR; ++m)
          if (m == lane) v = acc[m];
        const int n = r0 + i;
        if (b1) v += b1[n];
        if (b2) v += b2[n];
        if (b3) v += b3[n];
        if (relu) v = fmaxf(v, 0.f);
        Y[static_cast<size_t>(lane) * ldy + n] = v;
      }
    }
  }
  if (sm_out != nullptr) {
    // fused row softmax: the last CTA to publish its rows normalises every output row
    __shared__ int sm_last;
    __shared__ float sm_red[9];
    __threadfence();
    __syncthreads();
    if (tid == 0) sm_last = atomicAdd(sm_counter, 1u) == gridDim.x - 1;
    __syncthreads();
    if (sm_last) {
      __threadfence();
      for (int m = 0; m < M; ++m) {
        const float* yr = Y + static_cast<size_t>(m) * ldy;
        float mx = -INFINITY;
        for (int n = tid; n < N; n += 288) mx = fmaxf(mx, __ldcg(yr + n));
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        if (lane == 0) sm_red[warp] = mx;
        __syncthreads();
        mx = sm_red[0];
#pragma unroll
        for (int w = 1; w < 9; ++w) mx = fmaxf(mx, sm_red[w]);
        __syncthreads();
        float sum = 0.f;
        for (int n = tid; n < N; n += 288) sum += expf(__ldcg(yr + n) - mx);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
        if (lane == 0) sm_red[warp] = sum;
        __syncthreads();
        sum = sm_red[0];
#pragma unroll
        for (int w = 1; w < 9; ++w) sum += sm_red[w];
        __syncthreads();
        float* orow = sm_out + static_cast<size_t>(m) * sm_ldo;
        for (int n = tid; n < N; n += 288) orow[n] = expf(__ldcg(yr + n) - mx) / sum;
      }
      if (tid == 0) *sm_counter = 0u;
    }
  }
}

// Same contraction with plain vectorised loads (no smem ring): warp w of the grid takes rows
// w, w + #warps, ...; lane j loads float4 j, j + 32, ... of the row, 8 loads in flight, with
// an L2 cache-policy hint (ld.global.nc.L2::cache_hint) so kept weights land in the persisting
// set-aside (TMA bulk copies do not honour it on B200, Q29).  SF_GEMV_ROWS=ldg.
template <int MR>
__global__ void __launch_bounds__(256)
gemv_rows_ldg_kernel(const float* __restrict__ Bm, const float* __restrict__ X, float* __restrict__ Y,
                     int M, int N, int K, int ldb, int ldx, int ldy,
                     const float* __restrict__ b1, const float* __restrict__ b2,
                     const float* __restrict__ b3, int relu, int l2_hint,
                     float* __restrict__ sm_out, int sm_ldo, unsigned* __restrict__ sm_counter) {
  extern __shared__ __align__(16) float gl_xs[];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  sfdev::griddep_launch();
  sfdev::griddep_wait();
  for (int i = tid; i < MR * K; i += 256) {
    const int m = i / K, k = i % K;
    gl_xs[i] = m < M ? X[static_cast<size_t>(m) * ldx + k] : 0.f;
  }
  __syncthreads();
  const uint64_t pol = sfdev::l2_policy(l2_hint ? l2_hint : 2);
  const int nq = K / 4;
  const float4* x4 = reinterpret_cast<const float4*>(gl_xs);
  const int nwarps = gridDim.x * 8;
  for (int n = blockIdx.x * 8 + warp; n < N; n += nwarps) {
    const float4* w4 = reinterpret_cast<const float4*>(Bm + static_cast<size_t>(n) * ldb);
    float acc[MR];
#pragma unroll
    for (int m = 0; m < MR; ++m) acc[m] = 0.f;
    int q = lane;
    for (; q + 7 * 32 < nq; q += 8 * 32) {
      float4 w[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) w[u] = sfdev::ldg4_hint(w4 + q + 32 * u, pol);
#pragma unroll
      for (int u = 0; u < 8; ++u)
#pragma unroll
        for (int m = 0; m < MR; ++m) {
          const float4 xv = x4[m * nq + q + 32 * u];
          acc[m] = fmaf(xv.x, w[u].x, acc[m]);
          acc[m] = fmaf(xv.y, w[u].y, acc[m]);
          acc[m] = fmaf(xv.z, w[u].z, acc[m]);
          acc[m] = fmaf(xv.w, w[u].w, acc[m]);
        }
    }
    for (; q < nq; q += 32) {
      const float4 w = sfdev::ldg4_hint(w4 + q, pol);
#pragma unroll
      for (int m = 0; m < MR; ++m) {
        const float4 xv = x4[m * nq + q];
        acc[m] = fmaf(xv.x, w.x, acc[m]);
        acc[m] = fmaf(xv.y, w.y, acc[m]);
        acc[m] = fmaf(xv.z, w.z, acc[m]);
        acc[m] = fmaf(xv.w, w.w, acc[m]);
      }
    }
#pragma unroll
    for (int m = 0; m < MR; ++m)
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) acc[m] += __shfl_xor_sync(0xffffffffu, acc[m], o);
    if (lane < MR && lane < M) {
      float v = 0.f;
#pragma unroll
      for (int m = 0; m < MR; ++m)
        if (m == lane) v = acc[m];
      if (b1) v += b1[n];
      if (b2) v += b2[n];
      if (b3) v += b3[n];
      if (relu) v = fmaxf(v, 0.f);
      Y[static_cast<size_t>(lane) * ldy + n] = v;
    }
  }
  if (sm_out != nullptr) {
    __shared__ int sm_last;
    __shared__ float sm_red[8];
    __threadfence();
    __syncthreads();
    if (tid == 0) sm_last = atomicAdd(sm_counter, 1u) == gridDim.x - 1;
    __syncthreads();
    if (sm_last) {
      __threadfence();
      for (int m = 0; m < M; ++m) {
        const float* yr = Y + static_cast<size_t>(m) * ldy;
        float mx = -INFINITY;
        for (int n = tid; n < N; n += 256) mx = fmaxf(mx, __ldcg(yr + n));
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        if (lane == 0) sm_red[warp] = mx;
        __syncthreads();
        mx = sm_red[0];
#pragma unroll
        for (int w = 1; w < 8; ++w) mx = fmaxf(mx, sm_red[w]);
        __syncthreads();
        float sum = 0.f;
        for (int n = tid; n < N; n += 256) sum += expf(__ldcg(yr + n) - mx);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
        if (lane == 0) sm_red[warp] = sum;
        __syncthreads();
        sum = sm_red[0];
#pragma unroll
        for (int w = 1; w < 8; ++w) sum += sm_red[w];
        __syncthreads();
        float* orow = sm_out + static_cast<size_t>(m) * sm_ldo;
        for (int n = tid; n < N; n += 256) orow[n] = expf(__ldcg(yr + n) - mx) / sum;
      }
      if (tid == 0) *sm_counter = 0u;
    }
  }
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

thread_local bool g_cluster_used = false;  // the last launch_tma_t reduced its split-K in-kernel

template <int BN, bool AM, bool BMn, bool RAW, int BKT = BK, bool ATM = false>
cudaError_t launch_tma_t(const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& c,
                         const TParams& p, dim3 grid, cudaStream_t st) {
  auto kern = gemm_tma_kernel<BN, AM, BMn, RAW, BKT, ATM>;
  using TC = TCfg<BN, BKT, ATM>;
  static std::atomic<uint64_t> configured{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (!(configured.load() & bit)) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, TC::SMEM);
    if (e != cudaSuccess) return e;
    configured.fetch_or(bit);
  }
  const int smem = p.stages * TC::STAGE_BYTES + 1024 + 256;
  g_cluster_used = false;
  if (p.cluster_reduce) {
    // all tiles' clusters must be co-resident in one wave (clusters of S one-CTA-per-SM CTAs
    // leave GPC remainders idle: 36 clusters of 4 need a second wave on 148 SMs); otherwise
    // the workspace + reduce-kernel path runs instead
    static std::mutex mu;
    static std::map<std::tuple<int, int, int>, int> cap;  // (device, S, smem) -> max active clusters
    int dev = 0;
    cudaGetDevice(&dev);
    int ncl = 0;
    {
      std::lock_guard<std::mutex> lk(mu);
      auto key = std::make_tuple(dev, p.splits, smem);
      auto it = cap.find(key);
      if (it == cap.end()) {
        cudaLaunchConfig_t oc = {};
        oc.gridDim = grid;
        oc.blockDim = dim3(kThreads);
        oc.dynamicSmemBytes = smem;
        cudaLaunchAttribute oa[1];
        oa[0].id = cudaLaunchAttributeClusterDimension;
        oa[0].val.clusterDim.x = 1;
        oa[0].val.clusterDim.y = 1;
        oa[0].val.clusterDim.z = p.splits;
        oc.attrs = oa;
        oc.numAttrs = 1;
        if (cudaOccupancyMaxActiveClusters(&ncl, kern, &oc) != cudaSuccess) {
          cudaGetLastError();
          ncl = 0;
        }
        cap[key] = ncl;
      } else {
        ncl = it->second;
      }
    }
    if (static_cast<long>(grid.x) * grid.y > ncl) {
      TParams q = p;
      q.cluster_reduce = 0;
      kern<<<grid, kThreads, smem, st>>>(a, b, c, q);
      count_launch();
      return cudaGetLastError();
    }
    g_cluster_used = true;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = dim3(kThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 1;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = p.splits;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, a, b, c, p);
    count_launch();
    return e;
  }
  kern<<<grid, kThreads, smem, st>>>(a, b, c, p);
  count_launch();
  return cudaGetLastError();
}


template <int BN, bool RAW, int BKT = BK, bool ATM = false>
cudaError_t dispatch_major(bool a_mn, bool b_mn, const CUtensorMap& a, const CUtensorMap& b,
                           const CUtensorMap& c, const TParams& p, dim3 grid, cudaStream_t st) {
  if (a_mn && b_mn) return launch_tma_t<BN, true, true, RAW, BKT, ATM>(a, b, c, p, grid, st);
  if (a_mn) return launch_tma_t<BN, true, false, RAW, BKT, ATM>(a, b, c, p, grid, st);
  if (b_mn) return launch_tma_t<BN, false, true, RAW, BKT, ATM>(a, b, c, p, grid, st);
  return launch_tma_t<BN, false, false, RAW, BKT, ATM>(a, b, c, p, grid, st);
}


// SF_GEMV_PF=1: prefetch each CTA's weight slice into L2 up front (measured: 46 -> 50 us on
// the C4 chain with a dirty cold L2, 38.4 -> 40 us warm; off by default, Q33)
bool gemv_prefetch() {
  static const bool on = std::getenv("SF_GEMV_PF") && std::getenv("SF_GEMV_PF")[0] == '1';
  return on;
}

template <int MR, int BC>
cudaError_t launch_gemv_t(const CUtensorMap& w, const GemmArgs& a, int kper, cudaStream_t st) {
  auto kern = gemv_tma_kernel<MR, BC>;
  const size_t smem = GvCfg<MR, BC>::smem(kper);
  static std::atomic<uint64_t> configured{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (!(configured.load() & bit)) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         GvCfg<MR, BC>::smem(kGvMaxKper));
    if (e != cudaSuccess) return e;
    configured.fetch_or(bit);
  }
  const int grid = (a.N + BC - 1) / BC * kGvCluster;
  count_launch();
  return launch_k(kern, dim3(grid), dim3(288), smem, st, w, a.A, a.C, a.M, a.N, a.K, a.lda, a.ldc,
                  kper, a.acc ? 1 : 0, a.bias[0], a.bias[1], a.bias[2], a.relu ? 1 : 0,
                  a.b_const ? 1 : 0, a.l2_hint | (gemv_prefetch() ? kGvPrefetch : 0), a.sm_out, a.sm_ldo,
                  a.sm_counter, static_cast<const char*>(a.pf_next), a.pf_next ? a.pf_bytes : 0ull);
}

template <int BC>
cudaError_t dispatch_gemv_mr(const CUtensorMap& w, const GemmArgs& a, int kper, cudaStream_t st) {
  if (a.M == 1) return launch_gemv_t<1, BC>(w, a, kper, st);
  if (a.M == 2) return launch_gemv_t<2, BC>(w, a, kper, st);
  if (a.M <= 4) return launch_gemv_t<4, BC>(w, a, kper, st);
  return launch_gemv_t<8, BC>(w, a, kper, st);
}

}  // namespace

bool make_map2d(CUtensorMap* m, const void* base, uint64_t cols, uint64_t rows, uint64_t pitch_bytes,
                uint32_t box_cols, uint32_t box_rows, bool swizzle128) {
  return map2d(m, base, cols, rows, pitch_bytes, box_cols, box_rows,
               swizzle128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE);
}

bool gemv_tma_eligible(const GemmArgs& a) {
  auto al = [](const void* p) { return reinterpret_cast<uintptr_t>(p) % 16 == 0; };
  if (!encode_fn() || a.M < 1 || a.M > 8 || a.ta || a.tb) return false;
  if (a.N % 4 || a.ldb % 4 || a.ldc % 4 || !al(a.B) || !al(a.C)) return false;
  return (a.K + kGvCluster - 1) / kGvCluster <= kGvMaxKper;
}

bool gemv_rows_eligible(const GemmArgs& a) {
  auto al = [](const void* p) { return reinterpret_cast<uintptr_t>(p) % 16 == 0; };
  static const bool off = std::getenv("SF_GEMV_ROWS") && std::getenv("SF_GEMV_ROWS")[0] == '0';
  if (off || a.M < 1 || a.M > 8 || a.ta || !a.tb || a.acc) return false;
  if (a.K % 4 || a.ldb % 4 || a.K * 4 > kGrMaxRow || a.M * a.K * 4 > kGrMaxX || !al(a.B)) return false;
  return a.N > 0 && a.K > 0;
}

template <int MR>
cudaError_t launch_gemv_rows_ldg_t(const GemmArgs& a, cudaStream_t st) {
  auto kern = gemv_rows_ldg_kernel<MR>;
  const size_t smem = static_cast<size_t>(MR) * a.K * 4;
  static std::atomic<uint64_t> configured{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (!(configured.load() & bit)) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kGrMaxX);
    if (e != cudaSuccess) return e;
    configured.fetch_or(bit);
  }
  // 2 CTAs (16 warps) per SM, capped by one warp per row
  const int grid = std::max(1, std::min((a.N + 7) / 8, 2 * 148));
  count_launch();
  return launch_k(kern, dim3(grid), dim3(256), smem, st, a.B, a.A, a.C, a.M, a.N, a.K, a.ldb, a.lda,
                  a.ldc, a.bias[0], a.bias[1], a.bias[2], a.relu ? 1 : 0, a.l2_hint, a.sm_out,
                  a.sm_ldo, a.sm_counter);
}

template <int MR>
cudaError_t launch_gemv_rows_t(const GemmArgs& a, cudaStream_t st) {
  static const bool ldg = std::getenv("SF_GEMV_ROWS") && std::getenv("SF_GEMV_ROWS")[0] == 'l';
  if (ldg) return launch_gemv_rows_ldg_t<MR>(a, st);
  auto kern = gemv_rows_kernel<MR>;
  const int slot_f = (a.K + 31) / 32 * 32;
  const int slots = std::max(2, std::min(16, kGrRing / (slot_f * 4)));
  const size_t smem = static_cast<size_t>(slots) * slot_f * 4 + static_cast<size_t>(MR) * a.K * 4 +
                      2 * slots * 8 + 64;
  static std::atomic<uint64_t> configured{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = 1ull << (dev & 63);
  if (!(configured.load() & bit)) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         kGrRing + kGrMaxRow + kGrMaxX + 2 * 16 * 8 + 64);
    if (e != cudaSuccess) return e;
    configured.fetch_or(bit);
  }
  static int n_sms = [] {
    int d = 0, n = 148;
    cudaGetDevice(&d);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, d);
    return n;
  }();
  const int grid = std::min(a.N, n_sms);  // one CTA per SM: the next layer's CTA fits beside it
  count_launch();
  return launch_k(kern, dim3(grid), dim3(288), smem, st, a.B, a.A, a.C, a.M, a.N, a.K, a.ldb, a.lda,
                  a.ldc, slots, a.bias[0], a.bias[1], a.bias[2], a.relu ? 1 : 0, a.b_const ? 1 : 0,
                  a.l2_hint, a.sm_out, a.sm_ldo, a.sm_counter);
}

bool gemv_softmax_fusable(const GemmArgs& a) {
  static const char gemv_path = std::getenv("SF_GEMV") ? std::getenv("SF_GEMV")[0] : 't';
  static const bool off = std::getenv("SF_FUSE_SOFTMAX") && std::getenv("SF_FUSE_SOFTMAX")[0] == '0';
  if (off || a.acc) return false;
  if (a.tb) return gemv_rows_eligible(a);
  return gemv_path == 't' && gemv_tma_eligible(a);
}

cudaError_t launch_gemv_rows(const GemmArgs& a, cudaStream_t st) {
  if (a.M == 1) return launch_gemv_rows_t<1>(a, st);
  if (a.M == 2) return launch_gemv_rows_t<2>(a, st);
  if (a.M <= 4) return launch_gemv_rows_t<4>(a, st);
  return launch_gemv_rows_t<8>(a, st);
}

cudaError_t launch_gemv_tma(const GemmArgs& a, cudaStream_t st) {
  // widest column block that still puts one CTA on every SM
  int bc = 32;
  for (int c : {128, 64})
    if ((a.N + c - 1) / c * kGvCluster >= 148) { bc = c; break; }
  int kper = (a.K + kGvCluster - 1) / kGvCluster;
  kper = (kper + kGvRows - 1) / kGvRows * kGvRows;
  // the weight maps of an inference graph never change: encode once per (W, shape, box)
  struct Key {
    const void* p; int n, k, ld, bc;
    bool operator<(const Key& o) const {
      return std::tie(p, n, k, ld, bc) < std::tie(o.p, o.n, o.k, o.ld, o.bc);
    }
  };
  static std::mutex mu;
  static std::map<Key, CUtensorMap> cache;
  const Key key{a.B, a.N, a.K, a.ldb, bc};
  CUtensorMap w;
  {
    std::lock_guard<std::mutex> lk(mu);
    auto it = a.b_const ? cache.find(key) : cache.end();
    if (it != cache.end()) {
      w = it->second;
    } else {
      if (!map2d(&w, a.B, a.N, a.K, static_cast<uint64_t>(a.ldb) * 4, bc, kGvRows, CU_TENSOR_MAP_SWIZZLE_NONE))
        return cudaErrorInvalidValue;
      if (a.b_const && cache.size() < 4096) cache[key] = w;
    }
  }
  if (bc == 128) return dispatch_gemv_mr<128>(w, a, kper, st);
  if (bc == 64) return dispatch_gemv_mr<64>(w, a, kper, st);
  return dispatch_gemv_mr<32>(w, a, kper, st);
}

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
  // 128x256 tiles stage K in 16-deep blocks (4 stages instead of 2 in the same shared memory:
  // the 2-stage ring left the MMAs waiting on TMA latency); SF_GEMM_BK256=32 restores 32
  static const int bk256 = std::getenv("SF_GEMM_BK256") ? std::atoi(std::getenv("SF_GEMM_BK256")) : 16;
  const int bk = bn == 256 && bk256 == 16 && splits == 1 ? 16 : 32;
  const CUtensorMapSwizzle kK = bk == 16 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B;
  // A in TMEM (the default for the raw-hi kernels; SF_GEMM_ATM=0 keeps A in shared memory): an
  // MN-major A tile is then only read by the converters, so it lands as plain SWIZZLE_128B rows
  static const bool atm_env = !(std::getenv("SF_GEMM_ATM") && std::getenv("SF_GEMM_ATM")[0] == '0');
  const bool atm = atm_env && raw_hi;
  // split-K over 2..8 splits reduces inside the kernel (cluster of the tile's splits, DSMEM):
  // no workspace round trip, no reduce launch; SF_GEMM_CLUSTER_RED=0 keeps the workspace path
  static const bool cl_env = !(std::getenv("SF_GEMM_CLUSTER_RED") && std::getenv("SF_GEMM_CLUSTER_RED")[0] == '0');
  const bool cl_red = cl_env && splits >= 2 && splits <= 8 && bn <= 128 && a.ldc % 4 == 0 &&
                      reinterpret_cast<uintptr_t>(a.C) % 16 == 0;
  bool ok = a_mn ? map2d(&ma, a.A, a.M, a.K, static_cast<uint64_t>(a.lda) * 4, 32, bk,
                         atm ? CU_TENSOR_MAP_SWIZZLE_128B : kMN)
                 : map2d(&ma, a.A, a.K, a.M, static_cast<uint64_t>(a.lda) * 4, bk, BM, kK);
  // B: op(B) is K x N.  Stored [K][N] (MN-major) or [N][K] (TB, K-major).
  ok = ok && (b_mn ? map2d(&mb, a.B, a.N, a.K, static_cast<uint64_t>(a.ldb) * 4, 32, bk, kMN)
                   : map2d(&mb, a.B, a.K, a.N, static_cast<uint64_t>(a.ldb) * 4, bk, bn, kK));
  ok = ok && (splits == 1 ? map2d(&mc, a.C, a.N, a.M, static_cast<uint64_t>(a.ldc) * 4, 32, 32)
                          : map3d_ws(&mc, a.ws, a.N, a.M, splits));
  if (!ok) return cudaErrorInvalidValue;
  static const int dbg = std::getenv("SF_GEMM_DEBUG") ? std::atoi(std::getenv("SF_GEMM_DEBUG")) : 0;
  // ring depth: with more 128x64 tiles than SMs (no split-K), 2 stages let two CTAs share an SM, so
  // the grid runs in half the waves and one CTA's prologue / epilogue overlaps the other's
  // loads (tall forest GEMMs: 100352x64x148 41.9 -> 29.7 us, 25088x64x576 33.7 -> 27.6 us;
  // split-K shapes keep the deep ring).  SF_GEMM_STAGES overrides.
  static const int stages_env = std::getenv("SF_GEMM_STAGES") ? std::atoi(std::getenv("SF_GEMM_STAGES")) : -1;
  const int max_stages =
      atm ? (bn == 64 ? TCfg<64, 32, true>::STAGES : bn == 128 ? TCfg<128, 32, true>::STAGES
                                                                : bk == 16 ? TCfg<256, 16, true>::STAGES
                                                                           : TCfg<256, 32, true>::STAGES)
          : (bn == 64 ? TCfg<64>::STAGES : bn == 128 ? TCfg<128>::STAGES
                                                     : bk == 16 ? TCfg<256, 16>::STAGES : TCfg<256>::STAGES);
  int stages = max_stages;
  if (stages_env > 0) stages = std::min(stages_env, max_stages);
  else if (bn == 64 && (splits == 1 ? tiles_n * tiles_m > 148 : gemm_dual64())) stages = 2;  // 2 x 97 KB fit an SM
  // merged MMAs for 128x64 / 128x128 tiles (SF_GEMM_MERGE=0 disables): forest dW
  // 576x64x25088 33.1 -> 26.9 us, forward 25088x64x576 24.9 -> 22.9 us; C3 FFN forward
  // 512x4096x1024 35.6 -> 28.0 us, C3 iteration 67.8 -> 73.2 TFLOP/s
  static const bool merge_env = !(std::getenv("SF_GEMM_MERGE") && std::getenv("SF_GEMM_MERGE")[0] == '0');
  static const int merge_max = std::getenv("SF_GEMM_MERGE_BN") ? std::atoi(std::getenv("SF_GEMM_MERGE_BN")) : 128;
  const bool merge = atm && bn <= merge_max && merge_env;
  TParams p{a.M, a.N, a.K, a.ldc, splits, bk == 16 ? (a.K + 15) / 16 : kb_per_split, a.acc ? 1 : 0, dbg, stages,
            cl_red ? 1 : 0, merge ? 1 : 0, a.C, a.ws, a.counters};
  dim3 grid(tiles_n, tiles_m, splits);
  cudaError_t e;
  g_cluster_used = false;
  if (atm) {
    e = bn == 64    ? dispatch_major<64, true, 32, true>(a_mn, b_mn, ma, mb, mc, p, grid, st)
        : bn == 128 ? dispatch_major<128, true, 32, true>(a_mn, b_mn, ma, mb, mc, p, grid, st)
        : bk == 16  ? dispatch_major<256, true, 16, true>(a_mn, b_mn, ma, mb, mc, p, grid, st)
                    : dispatch_major<256, true, 32, true>(a_mn, b_mn, ma, mb, mc, p, grid, st);
  } else if (bn == 64)
    e = raw_hi ? dispatch_major<64, true>(a_mn, b_mn, ma, mb, mc, p, grid, st)
               : dispatch_major<64, false>(a_mn, b_mn, ma, mb, mc, p, grid, st);
  else if (bn == 256)
    e = bk == 16 ? dispatch_major<256, true, 16>(a_mn, b_mn, ma, mb, mc, p, grid, st)
                 : dispatch_major<256, true>(a_mn, b_mn, ma, mb, mc, p, grid, st);
  else
    e = raw_hi ? dispatch_major<128, true>(a_mn, b_mn, ma, mb, mc, p, grid, st)
               : dispatch_major<128, false>(a_mn, b_mn, ma, mb, mc, p, grid, st);
  if (e != cudaSuccess || splits == 1 || (cl_red && g_cluster_used)) return e;
  if (a.ldc % 4 || reinterpret_cast<uintptr_t>(a.C) % 16) return cudaErrorInvalidValue;
  const uint64_t total4 = static_cast<uint64_t>(a.M) * a.N / 4;
  splitk_reduce_kernel<<<static_cast<unsigned>((total4 + 31) / 32), 256, 0, st>>>(
      a.ws, a.C, a.M, a.N, splits, a.ldc, a.acc ? 1 : 0);
  count_launch();
  return cudaGetLastError();
}

}  // namespace sfk
