// Host-side launchers of the sm_100a kernels (internal to libswitchflow_b200.so).
// Every launcher is asynchronous on `st` and returns the cudaError_t of the launch.
#pragma once
#include <cstdint>
#include <cuda.h>
#include <cuda_runtime.h>

namespace sfk {

// Device-side copy descriptor of the multi-tensor walk: chunk_begin = prefix sum of
// span/16 over preceding descriptors; the array has n + 1 entries (sentinel holds the
// total chunk count).
struct DCopy {
  const uint8_t* src;
  uint8_t* dst;
  uint64_t nbytes;       // valid bytes copied (multiple of 4)
  uint64_t chunk_begin;  // first 16-B chunk of this descriptor in the flat chunk space
};

// Multi-tensor copy / pack / unpack / peer-store over a device descriptor array.
// patch_iter >= 0 overwrites bytes [16,24) of descriptor 0's destination (staging iter).
// tstamp (optional, device): {earliest CTA start, latest CTA end} in %globaltimer ns; the
// caller initialises it to {~0, 0}.
cudaError_t launch_mtcopy(const DCopy* d_descs, int n, uint64_t total_chunks,
                          int64_t patch_iter, cudaStream_t st, unsigned long long* tstamp = nullptr, int waves = 0);
cudaError_t launch_fill(void* dst, uint64_t n, uint8_t value, cudaStream_t st);
cudaError_t launch_copy2d(const void* src, uint64_t spitch, void* dst, uint64_t dpitch, uint64_t rows,
                          uint64_t width, cudaStream_t st);
// Single-buffer copy with pointer arguments (request I/O; 16-B aligned, nbytes % 4 == 0).
cudaError_t launch_copy(const void* src, void* dst, uint64_t nbytes, cudaStream_t st);
// The copy kernel launch_copy runs (kernel(const uint8_t* src, uint8_t* dst, uint64_t nbytes)):
// captured request graphs patch its pointers per request (cudaGraphExecKernelNodeSetParams).
const void* copy_kernel_fn();

// GEMM C[M,N] = op(A) op(B) (+C).  a_kcontig: A stored [M][K] (not transposed);
// b_kcontig: B stored [N][K] (i.e. TB).  ws / counters: split-K workspace (may be null
// when gemm_workspace_floats() == 0).  Deterministic (fixed split, fixed order).
struct GemmArgs {
  const float* A; const float* B; float* C;
  int M, N, K, lda, ldb, ldc;
  bool ta, tb, acc;
  float* ws; unsigned* counters;
  // optional fused epilogue (batch-1 GEMV path only): C = act(AB + b1 + b2 + b3)
  const float* bias[3] = {nullptr, nullptr, nullptr};
  bool relu = false;
  // B is not written by any kernel that may still be running (inference weights): the GEMV
  // may stream it before griddep_wait() under programmatic dependent launch
  bool b_const = false;
  // optional fused row softmax of the (epilogued) output into sm_out (TMA GEMV path only, see
  // gemv_softmax_fusable): the last column block to finish normalises every row; sm_counter is
  // a zeroed device counter the kernel leaves zeroed
  float* sm_out = nullptr;
  int sm_ldo = 0;
  unsigned* sm_counter = nullptr;
  // L2 policy of the GEMV weight stream: 0 default, 1 keep (evict_last: held in the persisting
  // L2 set-aside across requests), 2 stream (evict_first: do not displace kept weights)
  int l2_hint = 0;
  // TMA GEMV: constant weights of the NEXT layer (contiguous bytes) prefetched to L2 by this
  // kernel's CTAs once their own stream is issued (inference chains; nullptr = none)
  const void* pf_next = nullptr;
  uint64_t pf_bytes = 0;
  // constant B re-laid out in contiguous blocks (kernels_gemv.cu): the LDG-streamed GEMV
  const void* Bblk = nullptr;
  int blk_qw = 0, blk_kper = 0, blk_cl = 8;
};
// Blocked layout of a constant GEMV weight (kernels_gemv.cu)
struct GemvBlockPlan {
  bool ok = false;
  int qw = 0, kper = 0, n_cb = 0, cl = 8;  // cl: CTAs per column block (K split)
  uint64_t bytes = 0;
};
GemvBlockPlan plan_gemv_block(int M, int N, int K);
cudaError_t launch_gemv_block_layout(const float* W, void* Wb, int K, int N, int ldw, const GemvBlockPlan& p,
                                     cudaStream_t st);
bool gemv_blk_eligible(const GemmArgs& a);
cudaError_t launch_gemv_blk(const GemmArgs& a, cudaStream_t st);
bool gemv_softmax_fusable(const GemmArgs& a);
// M <= 8 with B stored [N][K] (TB, the inference weight layout): row-contiguous streaming GEMV
// with the same fused epilogue / softmax (kernels_gemm_tma.cu).
bool gemv_rows_eligible(const GemmArgs& a);
cudaError_t launch_gemv_rows(const GemmArgs& a, cudaStream_t st);
// True when launch_gemm can fuse a following BIAS_ACT into this GEMM's epilogue.
// Programmatic dependent launch for the launches this host thread makes (thread-local;
// the inference dispatcher enables it around a request's kernel chain).
void set_pdl(bool on);
bool pdl_enabled();

bool gemm_can_fuse_bias(int M, int N, int K, bool ta, bool tb, int ldb);
uint64_t gemm_workspace_floats(int M, int N, int K, bool ta, bool tb);
uint64_t gemm_counter_slots(int M, int N, int K, bool ta, bool tb);
cudaError_t launch_gemm(const GemmArgs& a, cudaStream_t st);
// The kernel path the calling thread's last launch_gemm took (diagnostics; sf_last_gemm_path).
enum GemmPathKind { kGemmTma = 1, kGemmLdg = 2, kGemvTma = 3, kGemvRows = 4, kGemvCluster = 5,
                    kGemvSplit = 6, kGemvPlain = 7, kGemvBlocked = 8 };
struct GemmPath { int kind = 0, bn = 0, splits = 0, a_mn = 0, b_mn = 0; };
GemmPath last_gemm_path();
// TMA-fed variant (kernels_gemm_tma.cu): needs 16-B aligned pointers and row pitches.
bool gemm_tma_eligible(const GemmArgs& a, int splits);
// M <= 8 (inference): TMA-streamed cluster GEMV with fused reduction + bias/ReLU epilogue.
bool gemv_tma_eligible(const GemmArgs& a);
bool make_map2d(CUtensorMap* m, const void* base, uint64_t cols, uint64_t rows, uint64_t pitch_bytes,
                uint32_t box_cols, uint32_t box_rows, bool swizzle128);

// Fused batch-M (M <= 8) MLP chain: h_{l+1} = act(h_l W_l + b_l) for every layer (+ softmax)
// in one persistent kernel (kernels_chain.cu).  layer[l].x must be layer[l-1].y.  Layer 0 is
// read from w0t, a transposed copy W_0^T [N_0][K_0 rounded up to 4] (zero-padded) laid out by
// launch_chain_w0t_layout (chain_w0t_floats floats).
constexpr int kChainMaxLayers = 6;
struct ChainLayerArgs {
  const float* W; int ldw;
  const float* x; int ldx;
  float* y; int ldy;
  const float* b[3];
  int K, N;
  bool relu;
};
struct ChainArgs {
  int n_layers = 0, M = 0;
  ChainLayerArgs layer[kChainMaxLayers];
  bool softmax = false;
  float* sm_out = nullptr;
  int sm_n = 0, sm_ldi = 0, sm_ldo = 0;
  float* ws = nullptr;
  unsigned* counters = nullptr;  // zero before the first launch; the kernel re-zeroes them
  const float* w0t = nullptr;    // W_0^T (16-B aligned)
};
bool chain_eligible(const ChainArgs& a);
uint64_t chain_ws_floats(const ChainArgs& a);
uint64_t chain_counter_slots(const ChainArgs& a);
uint64_t chain_w0t_floats(int K, int N);
cudaError_t launch_chain_w0t_layout(const float* W, int ldw, int K, int N, float* Wt, cudaStream_t st);
cudaError_t launch_chain(const ChainArgs& a, cudaStream_t st);
// diagnostics: when set, every chain launch records per-CTA phase timestamps (u64 [SMs][64])
void set_chain_trace(void* dev_buf);
void* chain_trace_buffer();
cudaError_t launch_gemv_tma(const GemmArgs& a, cudaStream_t st);
bool gemm_dual64();  // 128x64 GEMM tiles: two CTAs per SM (split planner + ring depth)
cudaError_t launch_gemm_tma(const GemmArgs& a, int bn, int splits, int kb_per_split, int tiles_n,
                            int tiles_m, bool raw_hi, cudaStream_t st);

// Elementwise / reduction ops (deterministic).  ws / counters sized by *_ws().
uint64_t colsum_ws_floats(int rows, int cols);
uint64_t colsum_counter_slots(int rows, int cols);
// act: 0 identity, 1 ReLU, 2 GELU; pre (optional): u = z + biases
cudaError_t launch_bias_act(const float* z, const float* b1, const float* b2, const float* b3,
                            float* h, int rows, int cols, int act, cudaStream_t st,
                            float* pre = nullptr);
// s = colsum(dz); with a mask operand dz = act'(mask) * x: mode 1 ReLU (mask = h > 0),
// mode 2 GELU (mask = u)
cudaError_t launch_colsum(const float* x, const float* h_mask, float* dz, float* s, int rows,
                          int cols, float* ws, unsigned* counters, cudaStream_t st, int mode = 1);
uint64_t softmax_ce_ws_floats(int rows);
cudaError_t launch_softmax_ce(const float* logits, const int32_t* labels, float* loss,
                              float* dlogits, int rows, int cols, float* ws, unsigned* counter,
                              cudaStream_t st);
cudaError_t launch_softmax(const float* logits, float* probs, int rows, int cols,
                           cudaStream_t st);

struct SgdDesc { float* w; float* a; const float* g; uint64_t n; float lr, mu; uint64_t begin; };
struct AdamDesc {
  float* w; float* m; float* v; const float* g; uint64_t n; float lr, b1, b2, eps;
  uint64_t begin;
};
// Multi-tensor optimizer updates over device descriptor arrays (n + 1 entries, sentinel).
cudaError_t launch_sgd(const SgdDesc* d, int n, uint64_t total, cudaStream_t st);
cudaError_t launch_adam(const AdamDesc* d, int n, uint64_t total, const int32_t* step,
                        cudaStream_t st);
cudaError_t launch_feed(const void* pool, const int32_t* step, void* x, uint64_t x_bytes,
                        int64_t pool_period, cudaStream_t st);
cudaError_t launch_step_inc(int32_t* step, cudaStream_t st);
// Reads `bytes` of p (L2 eviction with clean lines; migration probe).
cudaError_t launch_read_flush(const void* p, uint64_t bytes, cudaStream_t st);
// Clock anchor: writes %globaltimer to dst (device-visible mapped pinned host memory).
cudaError_t launch_stamp(unsigned long long* dst, cudaStream_t st);

// Library-wide kernel launch counter (evidence of the native path).
void count_launch(uint64_t n = 1);
uint64_t launches();

}  // namespace sfk
