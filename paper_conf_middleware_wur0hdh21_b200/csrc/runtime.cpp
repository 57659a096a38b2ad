// SwitchFlow-on-B200 runtime: graph registry, partitioner, live-set analysis, per-device
// versions (CUDA graphs), preemption scheduler and migration engine behind include/sf.h.
//
// Paper mapping (PAPER.md = /root/reference/PAPER.md):
//  * graph / session partition into subgraphs ........ PAPER.md:279-291, 323-325 (s.2, 2.1)
//  * one executor version per device ................... PAPER.md:635-637, 665-667 (s.3.2)
//  * session order preserved, executors interleave ..... PAPER.md:669-673 (s.3.2)
//  * task suspension: dispatched kernels finish ........ PAPER.md:699-704 (s.3.3)
//  * graph reconstruction onto GPU2 / CPU .............. PAPER.md:705-716 (s.3.3)
//  * context saving + async state transfer ............. PAPER.md:734-761 (s.3.3)
//  * resumption, no work lost .......................... PAPER.md:750-754 (s.3.3)
//  * invariant 1: no co-running GPU executors .......... PAPER.md:794-806 (s.3.4)
//  * preempter starts immediately after submission ..... PAPER.md:808-814 (s.3.4)
//  * atomic-flag executor sync, 1-LOC priority ......... PAPER.md:904-909, 920-923 (s.4)
//  * CPU executors scheduled freely (host feeds) ....... PAPER.md:816-826 (s.3.4)
//  * input reuse: immutable shared copy, lockstep ...... PAPER.md:828-896 (s.3.4, Fig. 5)
// B200 choices are described in DESIGN.md: cut at subgraph boundaries with in-flight
// activations (reading Q1), one multi-tensor pack / unpack / peer-store launch per cut,
// stream-ordered resume of a pre-instantiated CUDA graph on the target.
#include <cuda.h>
#include <cuda_runtime.h>
#include <time.h>

#include <algorithm>
#include <cmath>
#include <array>
#include <atomic>
#include <condition_variable>
#include <cstring>
#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <set>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

#include "sf.h"
#include "sf_kernels.h"

namespace {
inline void cpu_relax() {
#if defined(__x86_64__) || defined(__i386__)
  __builtin_ia32_pause();
#else
  std::atomic_signal_fence(std::memory_order_seq_cst);
#endif
}

thread_local std::string g_err;

sf_status fail(sf_status s, const std::string& msg) {
  g_err = msg;
  return s;
}

#define SF_CK(call)                                                                  \
  do {                                                                               \
    cudaError_t e_ = (call);                                                         \
    if (e_ != cudaSuccess)                                                           \
      return fail(SF_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_));    \
  } while (0)

uint64_t now_ns() {
  timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return static_cast<uint64_t>(ts.tv_sec) * 1000000000ull + static_cast<uint64_t>(ts.tv_nsec);
}

constexpr uint64_t kAlign = 256;
uint64_t round_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

bool persistent(int kind) { return kind == SF_PARAM || kind == SF_SLOT || kind == SF_SCALAR_STATE; }
bool optimizer_op(int t) { return t == SF_OP_SGD_MOM || t == SF_OP_ADAM || t == SF_OP_STEP_INC; }

struct Tensor {
  int rows, cols, dtype, kind;
  uint64_t nbytes, offset;
};

// Per-device copy list uploaded to device memory (DCopy[n + 1], last = sentinel).
struct CopyList {
  sfk::DCopy* d = nullptr;
  int n = 0;
  uint64_t total_chunks = 0;
  uint64_t bytes = 0;  // live bytes moved
};

struct Binding {
  int slot = -1;
  bool remote = false;       // partner arena mapped over CUDA IPC (no versions, no staging)
  void* ipc_base = nullptr;  // cudaIpcOpenMemHandle mapping (closed at sf_destroy)
  int ipc_device = -1;
  uint8_t* arena = nullptr;
  uint8_t* staging = nullptr;
  uint8_t* host_staging = nullptr;      // pinned host (host pointer)
  uint8_t* host_staging_dev = nullptr;  // its device mapping
  std::vector<cudaGraphExec_t> versions;
  std::vector<uint64_t> version_kernels;  // kernel nodes per version (launch accounting)
  float* ws = nullptr;
  unsigned* counters = nullptr;
  std::vector<CopyList> pack, unpack, pack_zc, unpack_zc;
  std::map<int, std::vector<CopyList>> peer;  // target slot -> per cut
  std::vector<std::pair<uint64_t, uint64_t>> poison_ranges;  // non-DATASET arena ranges
  // padded-pitch copies of DATASET GEMM operands whose row pitch is not 16-B aligned (the
  // TMA tensor-map requirement); refreshed from the arena at sf_start_training
  std::map<int, std::pair<float*, int>> shadow;  // tensor id -> (copy, pitch in floats)
  std::map<int, void*> prepared;  // optimizer group first op -> uploaded descriptor array
  std::set<int> l2_keep;          // inference weights kept in the persisting L2 set-aside
  bool l2_planned = false;
  std::map<int, std::pair<float*, unsigned*>> chain_bufs;  // chain first op -> (ws, counters)
  // GEMM ops with a misaligned (non-DATASET) operand or output: padded-pitch scratch copies
  // refreshed inside the version graph (copy2d before / after the GEMM)
  struct PadBuf { float* p = nullptr; int pitch = 0; };
  std::map<int, std::array<PadBuf, 3>> gemm_pad;  // op index -> {A, B, C}
  // inference: constant GEMV weights re-laid out in contiguous blocks (kernels_gemv.cu), built at
  // the binding's first request (sf_refresh_constants rebuilds them after the weights change)
  std::map<int, std::pair<void*, sfk::GemvBlockPlan>> blocked;  // tensor id -> (copy, plan)
  // fused inference chain: layer-0 weights transposed (W_0^T, kernels_chain.cu), same lifetime
  std::map<int, float*> folded;  // tensor id -> W_0^T
  // the whole request chain as ONE graph launch (SF_INFER_GRAPH=1): captured once per binding
  // (at sf_refresh_constants) between two copy kernels whose src / dst are patched per request
  // (cudaGraphExecKernelNodeSetParams), so one capture serves every request buffer
  struct ReqGraph {
    int state = 0;  // 0 not built, 1 ready, -1 failed (direct launches)
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t exec = nullptr;
    cudaGraphNode_t in_node = nullptr, out_node = nullptr;
    dim3 in_grid, in_block, out_grid, out_block;
    uint64_t kernels = 0;
  } rg;
  bool blocked_ready = false;
  std::vector<void*> dev_allocs;
};

struct Feed;

struct Graph {
  std::string name;
  Feed* feed = nullptr;              // host input stage feeding this graph (sf_attach_feed)
  std::vector<uint32_t> feed_tids;   // fed tensor of each feed buffer
  int feed_member = -1;              // shared feed: member index (attach order)
  int priority = 0;
  std::vector<Tensor> T;
  std::vector<sf_op_desc> ops;
  bool partitioned = false;
  std::vector<std::pair<int, int>> parts;
  std::vector<std::vector<uint32_t>> live;
  std::vector<uint64_t> live_bytes, staging_total, payload_start;
  std::vector<std::vector<uint64_t>> payload_off;
  std::vector<std::vector<uint8_t>> header;  // per cut: bytes [0, payload_start)
  uint64_t arena_bytes = 0, staging_bytes = 0, persistent_bytes = 0, max_live = 0;
  uint64_t ws_floats = 0, counter_slots = 0;
  std::vector<std::unique_ptr<Binding>> bind;  // per slot
  int input_tid = -1, output_tid = -1;
  std::vector<char> op_written;  // tensor id -> some op of the graph writes it
};

constexpr int kInferOwner = 1 << 20;
constexpr int kMaxInflight = 4;
// timing-event ring per slot: twice the largest window, so a retired subgraph's events stay
// valid until its device interval is mapped (deferred off the dispatch path)
constexpr int kEvRing = 2 * kMaxInflight;
constexpr int kCkEvents = 8;  // per slot: [0, 4) D2H chunk ring, [4, 8) H2D chunk ring

struct Request {
  sf_req_id id;
  Graph* g;
  int dev;
  const void* in;
  void* out;
  uint64_t arrival, start = 0, end = 0;
  bool done = false;
  int preempted_job = -1;
  int64_t cut_iter = -1;
  int cut_k = -1;
  float device_us = -1.f;
  float launch_us = -1.f;
  float dispatch_us = -1.f;  // dispatch decision .. first enqueue (host)
  std::string error;
};

struct Slot {
  int id, cuda;
  bool remote = false;  // another process's device (arena mapped over CUDA IPC)
  cudaStream_t s_train = nullptr, s_infer = nullptr, s_mig = nullptr;
  cudaEvent_t ev_infer = nullptr;
  cudaEvent_t ev_i0 = nullptr;  // timing: request chain start (ev_infer marks its end)
  unsigned long long* tstamp = nullptr;  // device {start, end} x 2 (pack/peer, unpack)
  // Device clock anchors (reading Q37): a stamp kernel writes %globaltimer into mapped
  // pinned memory and a timing event is recorded right behind it; any timing event of this
  // device then maps to CLOCK_MONOTONIC as g + elapsed(anchor, event) + offset, where offset
  // ties the GPU timer to the host clock (host read before launch / after the value landed).
  struct Anchor {
    cudaEvent_t ev;
    uint64_t enq_ns;   // host time the anchor was enqueued
    uint64_t g_ns;     // GPU time (%globaltimer ns) of the anchor event
    int64_t offset_ns; // host = GPU + offset (stamp value seen at host time ~h1 - 1 us)
    uint64_t unc_ns;   // half that window
    // position on the slot's DEVICE timeline: chained exactly through the event timer,
    // D_i = D_{i-1} + elapsed(anchor_{i-1}, anchor_i) (D_0 = g_0), so device times taken
    // against different anchors are mutually consistent (their order is the GPU's order)
    double D = 0.0;
  };
  cudaStream_t s_clk = nullptr;
  unsigned long long* clk_host = nullptr;  // pinned, mapped
  unsigned long long* clk_dev = nullptr;
  std::mutex clk_m;
  std::deque<Anchor> anchors;

  // drain gate (cfg.drain_gate, reading Q38): pinned mapped words, own cache lines.
  // gate[0] = G: a queued subgraph with ticket t runs once (int32)(G - t) >= 0; the host holds
  // tickets >= t with G = t - 1.  gate[16] = A: the GPU writes t right before its wait on G.
  volatile uint32_t* gate = nullptr;
  CUdeviceptr gate_G = 0, gate_A = 0;
  uint32_t next_ticket = 1;  // per-slot launch tickets (rt->m)
  bool gate_held = false;
  uint64_t gate_valve = 0;  // holds released by the dispatcher's 5 ms safety valve (diagnostics)
  std::atomic<int> owner{-1};  // device token (atomic: the spinning dispatcher polls it)
  size_t l2_setaside = 0, l2_max_window = 0;  // persisting L2 for inference weights
  std::deque<Request*> q;
  std::atomic<int> qn{0};       // q.size(), readable without the runtime lock
  std::thread dispatcher;
  uint64_t persistent_bound = 0;
};

struct Job {
  sf_job_id id;
  Graph* g;
  int dev;
  int64_t iters;
  int auto_target;
  int home = 0;           // slot the job started on (migrate_home policy)
  uint64_t t_submit = 0;  // CLOCK_MONOTONIC at sf_start_training / sf_adopt_job
  int64_t it = 0;
  int k = 0;
  int state = SF_JOB_RUNNING;
  bool preempt_req = false, preempt_park = false;
  std::vector<sf_cut_request> sched;
  size_t sched_pos = 0;
  int preempt_target = 0;
  uint64_t t_req = 0;
  bool cut_ready = false;
  bool mig_enqueued = false;
  bool holds_token = false;
  // early launch (cfg.early_launch): the driver is between its gate check and the
  // registration of a launched subgraph (runtime lock released); last_ev = completion event
  // of the newest in-flight subgraph, n_inflight = subgraphs on the device
  bool launching = false;
  cudaEvent_t last_ev = nullptr;
  int n_inflight = 0;
  struct Infl { uint32_t ticket; bool gated; cudaEvent_t end; };
  std::deque<Infl> infl;  // in-flight subgraphs, oldest first (drain gate; rt->m)
  // drain gate: a request held this job's queued subgraphs and ran first; the job still
  // migrates to its auto_target at its next boundary (the preemption the request triggered),
  // even when the request already finished by then
  bool gate_cut_pending = false;
  uint64_t gate_t_req = 0;
  sf_cut_info cut{};
  bool resume_req = false;
  int resume_dev = -1;
  bool stop_req = false;
  bool stamp_resume = false;
  bool adopted_pending = false;  // first launch of an adopted job: stamp time, no copy stats
  // host tier: the pinned staging of slot parked_slot holds L_k of cut (parked_iter, parked_k)
  int parked_slot = -1, parked_k = -1;
  int64_t parked_iter = -1;
  int64_t n_repark = 0;
  int n_preempt = 0;
  uint64_t migrated = 0;
  double pack_us = 0, xfer_us = 0, unpack_us = 0;
  uint64_t last_stop = 0, last_resume = 0;
  std::string error;
  std::thread driver;
  std::vector<cudaEvent_t> ev_sub, ev_a, ev_b, ev_c, ev_r;  // per slot; ev_r: resume point
  std::vector<cudaEvent_t> ev_ring;  // [slot * kEvRing + i]: in-flight subgraph ends
  std::vector<cudaEvent_t> ev_start; // [slot * kEvRing + i]: their starts (device trace)
  std::vector<cudaEvent_t> ev_ck;    // [slot * kCkEvents + i]: host-tier copy chunks in flight
};

// Host input stage (sf_create_feed).  Ring slot s holds iteration slot_iter[s]; states:
// 0 free, 1 being filled, 2 ready (pinned host bytes, shared: also the immutable device copy).
// A slot returns to free once every consumer's S_0 (which copies it into the arena) retired.
struct Feed {
  sf_feed_id id = 0;
  sf_host_stage_fn fn = nullptr;
  void* user = nullptr;
  int n = 0, depth = 2, dev = -1;
  bool shared = false;
  std::vector<uint64_t> bytes, off;  // per fed buffer: size, offset inside a ring slot
  uint64_t stride = 0;
  uint8_t* host = nullptr;   // pinned [depth][stride]
  uint8_t* dbuf = nullptr;   // shared: device [depth][stride], the immutable copies
  cudaStream_t st = nullptr;
  std::vector<cudaEvent_t> ev;  // shared: per ring slot, its H2D into dbuf completed
  std::vector<int64_t> slot_iter;
  std::vector<int> slot_state;
  std::vector<uint32_t> consumed;  // shared: bit m = member m copied the slot (S_0 retired)
  std::vector<Graph*> members;
  std::vector<Job*> member_jobs;
  int64_t next_iter = 0;
  bool active = false, inline_mode = false, failed = false;
  std::string error;
  int64_t turn_it = 0;  // shared: lockstep cursor (iteration, member)
  int turn_m = 0;
  uint64_t gen = 0;     // bumped when a job (re)starts the feed: stale fills are discarded
  std::thread stager;
};

}  // namespace

struct sf_runtime {
  sf_config cfg{};
  std::vector<std::unique_ptr<Slot>> slots;
  std::vector<std::unique_ptr<Graph>> graphs;
  std::vector<std::unique_ptr<Job>> jobs;
  std::vector<std::unique_ptr<Feed>> feeds;
  std::unordered_map<sf_req_id, std::unique_ptr<Request>> reqs;
  sf_req_id next_req = 1;
  std::mutex m;
  std::condition_variable cv;
  bool shutting_down = false;
  std::atomic<bool> stop_spin{false};
  std::vector<sf_trace_event> trace;
  std::vector<std::pair<double, double>> trace_D;  // per trace event: device-timeline d0, d1 (NaN: none)
  std::thread clk;  // refreshes every local slot's device clock anchor (Slot::Anchor)
  size_t trace_cap = 1 << 16;
  size_t trace_dropped = 0;
};

namespace {

void push_trace(sf_runtime* rt, const sf_trace_event& e, double D0 = std::nan(""),
                double D1 = std::nan("")) {  // rt->m held
  if (rt->trace.size() < rt->trace_cap) {
    rt->trace.push_back(e);
    rt->trace_D.emplace_back(D0, D1);
  } else {
    ++rt->trace_dropped;
  }
}

// ---------------------------------------------------------------------------------------
// Graph validation (mirrors the oracle's rules, written independently from the paper).
// ---------------------------------------------------------------------------------------
sf_status validate(const Graph& g) {
  const int n = static_cast<int>(g.T.size());
  auto chk = [&](bool c, sf_status s, const std::string& msg) -> sf_status {
    return c ? SF_OK : fail(s, msg);
  };
  for (size_t j = 0; j < g.ops.size(); ++j) {
    const sf_op_desc& o = g.ops[j];
    const std::string at = "op " + std::to_string(j) + ": ";
    if (o.type < SF_OP_GEMM || o.type > SF_OP_STEP_INC)
      return fail(SF_EUNSUPPORTED, at + "op type outside the fixed op set");
    if (o.n_in < 0 || o.n_in > 6 || o.n_out < 0 || o.n_out > 3) return fail(SF_EINVAL, at + "arity");
    for (int i = 0; i < o.n_in; ++i)
      if (o.in[i] < 0 || o.in[i] >= n) return fail(SF_EINVAL, at + "input id out of range");
    for (int i = 0; i < o.n_out; ++i) {
      if (o.out[i] < 0 || o.out[i] >= n) return fail(SF_EINVAL, at + "output id out of range");
      const Tensor& t = g.T[o.out[i]];
      if (t.kind == SF_DATASET) return fail(SF_EINVAL, at + "writes a DATASET tensor");
      if (persistent(t.kind) && !optimizer_op(o.type))
        return fail(SF_EINVAL, at + "only optimizer ops write persistent state");
    }
    auto T = [&](int id) -> const Tensor& { return g.T[id]; };
    sf_status s = SF_OK;
    switch (o.type) {
      case SF_OP_GEMM: {
        if ((s = chk(o.n_in == 2 && o.n_out == 1, SF_EINVAL, at + "gemm arity"))) return s;
        const Tensor &A = T(o.in[0]), &B = T(o.in[1]), &C = T(o.out[0]);
        const int M = (o.flags & SF_GEMM_TA) ? A.cols : A.rows;
        const int K = (o.flags & SF_GEMM_TA) ? A.rows : A.cols;
        const int K2 = (o.flags & SF_GEMM_TB) ? B.cols : B.rows;
        const int N = (o.flags & SF_GEMM_TB) ? B.rows : B.cols;
        if ((s = chk(K == K2 && C.rows == M && C.cols == N && K > 0, SF_EINVAL, at + "gemm shapes"))) return s;
        if ((s = chk(A.dtype == SF_F32 && B.dtype == SF_F32 && C.dtype == SF_F32, SF_EUNSUPPORTED,
                     at + "gemm dtype")))
          return s;
        break;
      }
      case SF_OP_BIAS_ACT: {
        const bool gelu = o.flags & SF_ACT_GELU;
        if ((s = chk(o.n_in >= 2 && o.n_in <= 4 && (o.n_out == 1 || (gelu && o.n_out == 2)), SF_EINVAL,
                     at + "bias_act arity")))
          return s;
        if ((s = chk(!(gelu && (o.flags & SF_ACT_RELU)), SF_EINVAL, at + "one activation"))) return s;
        const Tensor &z = T(o.in[0]), &h = T(o.out[0]);
        if ((s = chk(z.rows == h.rows && z.cols == h.cols, SF_EINVAL, at + "bias_act shape"))) return s;
        if (o.n_out == 2 && (s = chk(T(o.out[1]).rows == z.rows && T(o.out[1]).cols == z.cols, SF_EINVAL,
                                     at + "bias_act pre-activation shape")))
          return s;
        for (int i = 1; i < o.n_in; ++i)
          if ((s = chk(T(o.in[i]).rows == 1 && T(o.in[i]).cols == z.cols, SF_EINVAL, at + "bias shape")))
            return s;
        break;
      }
      case SF_OP_BIAS_ACT_BWD: {
        if ((s = chk(o.n_in == 2 && o.n_out == 2, SF_EINVAL, at + "bias_act_bwd arity"))) return s;
        const Tensor &dh = T(o.in[0]), &h = T(o.in[1]), &dz = T(o.out[0]), &db = T(o.out[1]);
        if ((s = chk(dh.rows == h.rows && dh.cols == h.cols && dz.rows == h.rows && dz.cols == h.cols &&
                         db.rows == 1 && db.cols == h.cols,
                     SF_EINVAL, at + "bias_act_bwd shapes")))
          return s;
        break;
      }
      case SF_OP_COLSUM: {
        if ((s = chk(o.n_in == 1 && o.n_out == 1 && T(o.out[0]).rows == 1 &&
                         T(o.out[0]).cols == T(o.in[0]).cols,
                     SF_EINVAL, at + "colsum")))
          return s;
        break;
      }
      case SF_OP_SOFTMAX_CE: {
        if ((s = chk(o.n_in == 2 && o.n_out == 2, SF_EINVAL, at + "softmax_ce arity"))) return s;
        const Tensor &l = T(o.in[0]), &y = T(o.in[1]), &loss = T(o.out[0]), &d = T(o.out[1]);
        if ((s = chk(y.dtype == SF_I32 && y.rows == l.rows && y.cols == 1 && loss.rows == 1 &&
                         loss.cols == 1 && d.rows == l.rows && d.cols == l.cols,
                     SF_EINVAL, at + "softmax_ce shapes")))
          return s;
        break;
      }
      case SF_OP_SOFTMAX: {
        if ((s = chk(o.n_in == 1 && o.n_out == 1 && T(o.in[0]).rows == T(o.out[0]).rows &&
                         T(o.in[0]).cols == T(o.out[0]).cols,
                     SF_EINVAL, at + "softmax")))
          return s;
        break;
      }
      case SF_OP_SGD_MOM: {
        if ((s = chk(o.n_in == 1 && o.n_out == 2, SF_EINVAL, at + "sgd arity"))) return s;
        const Tensor &gr = T(o.in[0]), &w = T(o.out[0]), &a = T(o.out[1]);
        if ((s = chk(gr.rows == w.rows && gr.cols == w.cols && a.rows == w.rows && a.cols == w.cols,
                     SF_EINVAL, at + "sgd shapes")))
          return s;
        break;
      }
      case SF_OP_ADAM: {
        if ((s = chk(o.n_in == 2 && o.n_out == 3, SF_EINVAL, at + "adam arity"))) return s;
        const Tensor &gr = T(o.in[0]), &st = T(o.in[1]);
        for (int i = 0; i < 3; ++i)
          if ((s = chk(T(o.out[i]).rows == gr.rows && T(o.out[i]).cols == gr.cols, SF_EINVAL,
                       at + "adam shapes")))
            return s;
        if ((s = chk(st.dtype == SF_I32 && st.rows * st.cols == 1, SF_EINVAL, at + "adam step"))) return s;
        break;
      }
      case SF_OP_FEED: {
        if ((s = chk(o.n_in == 2 && o.n_out == 1, SF_EINVAL, at + "feed arity"))) return s;
        const Tensor &pool = T(o.in[0]), &st = T(o.in[1]), &x = T(o.out[0]);
        if ((s = chk(pool.kind == SF_DATASET && pool.cols == x.cols && x.rows > 0 &&
                         pool.rows % x.rows == 0 && pool.dtype == x.dtype && st.dtype == SF_I32,
                     SF_EINVAL, at + "feed shapes")))
          return s;
        break;
      }
      case SF_OP_STEP_INC: {
        if ((s = chk(o.n_out == 1 && T(o.out[0]).dtype == SF_I32, SF_EINVAL, at + "step_inc"))) return s;
        break;
      }
    }
  }
  // read-before-write within an iteration
  std::vector<char> written(n, 0), has_writer(n, 0);
  for (const auto& o : g.ops)
    for (int i = 0; i < o.n_out; ++i) has_writer[o.out[i]] = 1;
  for (size_t j = 0; j < g.ops.size(); ++j) {
    const sf_op_desc& o = g.ops[j];
    std::vector<int> reads(o.in, o.in + o.n_in);
    if (o.type == SF_OP_GEMM && (o.flags & SF_GEMM_ACC)) reads.push_back(o.out[0]);
    if (optimizer_op(o.type)) reads.insert(reads.end(), o.out, o.out + o.n_out);
    for (int t : reads) {
      const int k = g.T[t].kind;
      if (persistent(k) || k == SF_DATASET || written[t]) continue;
      if ((k == SF_INPUT || k == SF_LABEL) && !has_writer[t]) continue;
      return fail(SF_EINVAL, "op " + std::to_string(j) + ": reads tensor " + std::to_string(t) +
                                 " before it is written");
    }
    for (int i = 0; i < o.n_out; ++i) written[o.out[i]] = 1;
  }
  return SF_OK;
}

std::vector<int> op_reads(const sf_op_desc& o) {
  std::vector<int> r(o.in, o.in + o.n_in);
  if (o.type == SF_OP_GEMM && (o.flags & SF_GEMM_ACC)) r.push_back(o.out[0]);
  if (optimizer_op(o.type)) r.insert(r.end(), o.out, o.out + o.n_out);
  return r;
}

// Live set at cut k: persistent state, plus every tensor written
// before S_k that an op at/after S_k reads before overwriting it, plus OUTPUT tensors
// already produced (fetched at iteration end).  Externally fed INPUT/LABEL count as
// written at the start of S_0.
std::vector<uint32_t> compute_live(const Graph& g, int k) {
  const int start = g.parts[k].first;
  const int nT = static_cast<int>(g.T.size()), nO = static_cast<int>(g.ops.size());
  std::vector<char> written_before(nT, 0), has_writer(nT, 0);
  for (int j = 0; j < nO; ++j)
    for (int i = 0; i < g.ops[j].n_out; ++i) {
      has_writer[g.ops[j].out[i]] = 1;
      if (j < start) written_before[g.ops[j].out[i]] = 1;
    }
  // first access at/after start: +1 read first, -1 write first, 0 none
  std::vector<int> first(nT, 0);
  for (int j = start; j < nO; ++j) {
    const sf_op_desc& o = g.ops[j];
    for (int t : op_reads(o))
      if (first[t] == 0) first[t] = 1;
    for (int i = 0; i < o.n_out; ++i)
      if (first[o.out[i]] == 0) first[o.out[i]] = -1;
  }
  std::vector<uint32_t> live;
  for (int t = 0; t < nT; ++t) {
    const Tensor& x = g.T[t];
    if (persistent(x.kind)) { live.push_back(t); continue; }
    if (x.kind == SF_DATASET) continue;
    const bool fed_ext = (x.kind == SF_INPUT || x.kind == SF_LABEL) && !has_writer[t];
    const bool wb = written_before[t] || (fed_ext && start > 0);
    if (!wb) continue;
    if (x.kind == SF_OUTPUT || first[t] == 1) live.push_back(t);
  }
  return live;
}

sf_status do_partition(Graph& g, const sf_partition_opts& o) {
  g.parts.clear();
  std::vector<std::pair<int, int>> runs;
  int s = 0;
  const int nO = static_cast<int>(g.ops.size());
  for (int j = 1; j <= nO; ++j)
    if (j == nO || g.ops[j].phase != g.ops[s].phase) {
      runs.emplace_back(s, j);
      s = j;
    }
  if (o.update_chunks > 1) {
    std::vector<std::pair<int, int>> split;
    for (auto [a, b] : runs) {
      bool opt = false;
      for (int j = a; j < b; ++j) opt |= optimizer_op(g.ops[j].type);
      uint64_t W = 0;
      for (int j = a; j < b; ++j)
        if (g.ops[j].type == SF_OP_SGD_MOM || g.ops[j].type == SF_OP_ADAM) W += g.T[g.ops[j].out[0]].nbytes;
      if (!opt || W == 0) { split.emplace_back(a, b); continue; }
      const uint64_t U = static_cast<uint64_t>(o.update_chunks);
      uint64_t c = 0;
      int start = a;
      int64_t prev = -1;
      for (int j = a; j < b; ++j) {
        const int64_t ch = static_cast<int64_t>(std::min<uint64_t>(U - 1, (U * c) / W));
        if (prev >= 0 && ch != prev) { split.emplace_back(start, j); start = j; }
        prev = ch;
        if (g.ops[j].type == SF_OP_SGD_MOM || g.ops[j].type == SF_OP_ADAM) c += g.T[g.ops[j].out[0]].nbytes;
      }
      split.emplace_back(start, b);
    }
    runs = std::move(split);
  }
  if (o.policy == SF_PART_PER_LAYER_PHASE) {
    g.parts = runs;
  } else if (o.policy == SF_PART_MAX_OPS && o.max_ops > 0) {
    for (auto [a, b] : runs) {
      bool opt = false;
      for (int j = a; j < b; ++j) opt |= optimizer_op(g.ops[j].type);
      if (opt) { g.parts.emplace_back(a, b); continue; }
      for (int c = a; c < b; c += o.max_ops) g.parts.emplace_back(c, std::min(b, c + o.max_ops));
    }
  } else {
    return fail(SF_EINVAL, "unknown partition policy");
  }
  // arena layout: every tensor at a 256-B aligned offset, ascending id
  uint64_t off = 0;
  g.persistent_bytes = 0;
  for (auto& t : g.T) {
    t.offset = off;
    off += round_up(std::max<uint64_t>(t.nbytes, 1), kAlign);
    if (persistent(t.kind)) g.persistent_bytes += t.nbytes;
  }
  g.arena_bytes = off;
  const int n = static_cast<int>(g.parts.size());
  g.live.assign(n, {});
  g.live_bytes.assign(n, 0);
  g.staging_total.assign(n, 0);
  g.payload_start.assign(n, 0);
  g.payload_off.assign(n, {});
  g.header.assign(n, {});
  g.staging_bytes = 0;
  g.max_live = 0;
  for (int k = 0; k < n; ++k) {
    g.live[k] = compute_live(g, k);
    const auto& L = g.live[k];
    // staging format: 32-B header, 24-B entries, payloads at 256-B offsets
    const uint64_t ps = round_up(32 + 24 * static_cast<uint64_t>(L.size()), kAlign);
    uint64_t p = ps, bytes = 0;
    std::vector<uint64_t> offs;
    for (uint32_t t : L) {
      offs.push_back(p);
      p += round_up(g.T[t].nbytes, kAlign);
      bytes += g.T[t].nbytes;
    }
    std::vector<uint8_t> h(ps, 0);
    auto put32 = [&](size_t at, uint32_t v) { std::memcpy(&h[at], &v, 4); };
    auto put64 = [&](size_t at, uint64_t v) { std::memcpy(&h[at], &v, 8); };
    std::memcpy(&h[0], "SFST", 4);
    put32(4, 1);
    put32(8, static_cast<uint32_t>(L.size()));
    put32(12, static_cast<uint32_t>(k));
    put64(16, 0);  // iter, patched by the pack kernel
    put64(24, p);
    for (size_t e = 0; e < L.size(); ++e) {
      put32(32 + 24 * e, L[e]);
      put32(36 + 24 * e, static_cast<uint32_t>(g.T[L[e]].dtype));
      put64(40 + 24 * e, offs[e]);
      put64(48 + 24 * e, g.T[L[e]].nbytes);
    }
    g.header[k] = std::move(h);
    g.payload_start[k] = ps;
    g.payload_off[k] = std::move(offs);
    g.staging_total[k] = p;
    g.live_bytes[k] = bytes;
    g.staging_bytes = std::max(g.staging_bytes, p);
    g.max_live = std::max(g.max_live, bytes);
  }
  // workspace: max over ops (ops of one subgraph run sequentially on one stream)
  g.ws_floats = 0;
  g.counter_slots = 1;
  for (const auto& op : g.ops) {
    if (op.type == SF_OP_GEMM) {
      const Tensor &A = g.T[op.in[0]], &B = g.T[op.in[1]];
      const bool ta = op.flags & SF_GEMM_TA, tb = op.flags & SF_GEMM_TB;
      const int M = ta ? A.cols : A.rows, K = ta ? A.rows : A.cols, N = tb ? B.rows : B.cols;
      g.ws_floats = std::max(g.ws_floats, sfk::gemm_workspace_floats(M, N, K, ta, tb));
      g.counter_slots = std::max(g.counter_slots, sfk::gemm_counter_slots(M, N, K, ta, tb));
    } else if (op.type == SF_OP_BIAS_ACT_BWD || op.type == SF_OP_COLSUM) {
      const Tensor& x = g.T[op.in[0]];
      g.ws_floats = std::max(g.ws_floats, sfk::colsum_ws_floats(x.rows, x.cols));
      g.counter_slots = std::max(g.counter_slots, sfk::colsum_counter_slots(x.rows, x.cols));
    } else if (op.type == SF_OP_SOFTMAX_CE) {
      g.ws_floats = std::max(g.ws_floats, sfk::softmax_ce_ws_floats(g.T[op.in[0]].rows));
    }
  }
  g.counter_slots += 1;  // the last slot: completion counter of a GEMV with fused softmax
  g.partitioned = true;
  return SF_OK;
}

// ---------------------------------------------------------------------------------------
// Version build: launch the ops of subgraph k for one binding (captured into a CUDA graph).
// ---------------------------------------------------------------------------------------
struct Capture {
  Graph& g;
  Binding& b;
  cudaStream_t st;
  bool dry;                          // prepare pass: upload descriptor arrays, launch nothing
  std::map<int, void*>* prepared;    // first op index of an optimizer group -> device array
  const std::set<int>* l2_keep = nullptr;  // weights held in the persisting L2 set-aside
  // request I/O in place (direct inference launches): the INPUT tensor is read from, and the
  // OUTPUT tensor written to, the caller's buffers instead of arena copies
  int redir_in = -1, redir_out = -1;
  uint8_t* in_ptr = nullptr;
  uint8_t* out_ptr = nullptr;
  uint8_t* ptr(int t) const {
    if (t == redir_in) return in_ptr;
    if (t == redir_out) return out_ptr;
    return b.arena + g.T[t].offset;
  }
  float* f(int t) const { return reinterpret_cast<float*>(ptr(t)); }
};

sf_status upload(Binding& b, const void* host, size_t bytes, void** out) {
  void* d = nullptr;
  SF_CK(cudaMalloc(&d, std::max<size_t>(bytes, 16)));
  SF_CK(cudaMemcpy(d, host, bytes, cudaMemcpyHostToDevice));
  b.dev_allocs.push_back(d);
  *out = d;
  return SF_OK;
}

// Fused inference chain (kernels_chain.cu): GEMM(M <= 8, constant B) [-> BIAS_ACT] -> GEMM
// [-> BIAS_ACT] ... [-> SOFTMAX] inside [j, e), each GEMM reading the previous layer's output.
// Returns the number of ops covered (0 = no chain of >= 2 layers starts at j).
int match_chain(Capture& c, int j, int e, sfk::ChainArgs* out) {
  // opt-in (SF_CHAIN=1): the fused chain is parity-green, but on the C4 model the per-layer
  // GEMV kernels under programmatic dependent launch measure faster (reading Q42:
  // its two global reductions + softmax add a ~12 us serial tail after the weight stream)
  static const bool enabled = std::getenv("SF_CHAIN") && std::getenv("SF_CHAIN")[0] == '1';
  if (!enabled) return 0;
  Graph& g = c.g;
  sfk::ChainArgs a;
  int i = j, prev_y = -1, w0 = -1;
  auto readers = [&](int t) {
    int n = 0;
    for (const auto& q : g.ops)
      for (int r : op_reads(q)) n += (r == t);
    return n;
  };
  while (i < e && a.n_layers < sfk::kChainMaxLayers) {
    const sf_op_desc& o = g.ops[i];
    if (o.type != SF_OP_GEMM || (o.flags & (SF_GEMM_TA | SF_GEMM_TB | SF_GEMM_ACC))) break;
    const Tensor &A = g.T[o.in[0]], &B = g.T[o.in[1]], &C = g.T[o.out[0]];
    if (C.rows > 8 || g.op_written[o.in[1]] || c.b.shadow.count(o.in[1]) || c.b.gemm_pad.count(i)) break;
    if (a.n_layers > 0 && (o.in[0] != prev_y || C.rows != a.M)) break;
    sfk::ChainLayerArgs& L = a.layer[a.n_layers];
    L = sfk::ChainLayerArgs{};
    if (a.n_layers == 0) w0 = o.in[1];
    L.W = c.f(o.in[1]); L.ldw = B.cols;
    L.x = c.f(o.in[0]); L.ldx = A.cols;
    L.K = A.cols; L.N = C.cols;
    int y = o.out[0], used = 1;
    if (i + 1 < e && g.ops[i + 1].type == SF_OP_BIAS_ACT && g.ops[i + 1].in[0] == o.out[0] &&
        !(g.ops[i + 1].flags & SF_ACT_GELU) && C.kind != SF_OUTPUT && readers(o.out[0]) == 1) {
      const sf_op_desc& ba = g.ops[i + 1];
      for (int q = 1; q < ba.n_in; ++q) L.b[q - 1] = c.f(ba.in[q]);
      L.relu = ba.flags & SF_ACT_RELU;
      y = ba.out[0];
      used = 2;
    }
    L.y = c.f(y); L.ldy = g.T[y].cols;
    a.M = C.rows;
    ++a.n_layers;
    prev_y = y;
    i += used;
  }
  if (a.n_layers < 2) return 0;
  if (i < e && g.ops[i].type == SF_OP_SOFTMAX && g.ops[i].in[0] == prev_y) {
    const Tensor& P = g.T[g.ops[i].out[0]];
    a.softmax = true;
    a.sm_out = c.f(g.ops[i].out[0]);
    a.sm_n = P.cols;
    a.sm_ldi = g.T[prev_y].cols;
    a.sm_ldo = P.cols;
    ++i;
  }
  if (!sfk::chain_eligible(a)) return 0;
  auto fw = c.b.folded.find(w0);
  if (fw == c.b.folded.end()) {  // W_0^T: allocated in the prepare pass, laid out by layout_blocked
    if (!c.dry) return 0;
    void* d = nullptr;
    const Tensor& W0 = g.T[w0];
    if (cudaMalloc(&d, sfk::chain_w0t_floats(W0.rows, W0.cols) * sizeof(float)) != cudaSuccess) {
      cudaGetLastError();
      return 0;
    }
    c.b.dev_allocs.push_back(d);
    fw = c.b.folded.emplace(w0, static_cast<float*>(d)).first;
    c.b.blocked_ready = false;
  }
  a.w0t = fw->second;
  *out = a;
  return i - j;
}

sf_status launch_subgraph_ops(Capture& c, int k) {
  Graph& g = c.g;
  const auto [a, e] = g.parts[k];
  int j = a;
  while (j < e) {
    const sf_op_desc& o = g.ops[j];
    cudaError_t err = cudaSuccess;
    if (o.type == SF_OP_SGD_MOM) {
      const int first = j;
      std::vector<sfk::SgdDesc> ds;
      uint64_t q = 0;
      while (j < e && g.ops[j].type == SF_OP_SGD_MOM) {
        const sf_op_desc& s = g.ops[j];
        sfk::SgdDesc d{c.f(s.out[0]), c.f(s.out[1]), c.f(s.in[0]),
                       static_cast<uint64_t>(g.T[s.out[0]].rows) * g.T[s.out[0]].cols, s.f[0], s.f[1], q};
        q += (d.n + 3) / 4;
        ds.push_back(d);
        ++j;
      }
      sfk::SgdDesc sent{};
      sent.begin = q;
      ds.push_back(sent);
      void* dd;
      if (c.dry) {
        if (sf_status s = upload(c.b, ds.data(), ds.size() * sizeof(sfk::SgdDesc), &dd)) return s;
        (*c.prepared)[first] = dd;
        continue;
      }
      dd = (*c.prepared)[first];
      err = sfk::launch_sgd(static_cast<sfk::SgdDesc*>(dd), static_cast<int>(ds.size()) - 1, q, c.st);
      if (err != cudaSuccess) return fail(SF_ECUDA, std::string("sgd: ") + cudaGetErrorString(err));
      continue;
    }
    if (o.type == SF_OP_ADAM) {
      const int first = j;
      std::vector<sfk::AdamDesc> ds;
      uint64_t q = 0;
      const int step_t = o.in[1];
      while (j < e && g.ops[j].type == SF_OP_ADAM && g.ops[j].in[1] == step_t) {
        const sf_op_desc& s = g.ops[j];
        sfk::AdamDesc d{c.f(s.out[0]), c.f(s.out[1]), c.f(s.out[2]), c.f(s.in[0]),
                        static_cast<uint64_t>(g.T[s.out[0]].rows) * g.T[s.out[0]].cols,
                        s.f[0], s.f[1], s.f[2], s.f[3], q};
        q += (d.n + 3) / 4;
        ds.push_back(d);
        ++j;
      }
      sfk::AdamDesc sent{};
      sent.begin = q;
      ds.push_back(sent);
      void* dd;
      if (c.dry) {
        if (sf_status s = upload(c.b, ds.data(), ds.size() * sizeof(sfk::AdamDesc), &dd)) return s;
        (*c.prepared)[first] = dd;
        continue;
      }
      dd = (*c.prepared)[first];
      err = sfk::launch_adam(static_cast<sfk::AdamDesc*>(dd), static_cast<int>(ds.size()) - 1, q,
                             reinterpret_cast<const int32_t*>(c.ptr(step_t)), c.st);
      if (err != cudaSuccess) return fail(SF_ECUDA, std::string("adam: ") + cudaGetErrorString(err));
      continue;
    }
    if (o.type == SF_OP_GEMM) {
      sfk::ChainArgs ca;
      const int n_ops = match_chain(c, j, e, &ca);
      if (n_ops > 0) {
        auto& buf = c.b.chain_bufs[j];
        if (c.dry) {
          if (!buf.first) {
            void *w = nullptr, *cn = nullptr;
            const uint64_t wf = sfk::chain_ws_floats(ca), cs = sfk::chain_counter_slots(ca);
            if (cudaMalloc(&w, std::max<uint64_t>(wf, 4) * 4) != cudaSuccess || cudaMalloc(&cn, cs * 4) != cudaSuccess ||
                cudaMemset(cn, 0, cs * 4) != cudaSuccess)
              return fail(SF_ENOMEM, "chain workspace");
            c.b.dev_allocs.push_back(w);
            c.b.dev_allocs.push_back(cn);
            buf = {static_cast<float*>(w), static_cast<unsigned*>(cn)};
          }
          j += n_ops;
          continue;
        }
        ca.ws = buf.first;
        ca.counters = buf.second;
        if (!ca.counters) return fail(SF_ESTATE, "chain workspace not prepared");
        err = sfk::launch_chain(ca, c.st);
        if (err != cudaSuccess) return fail(SF_ECUDA, "op " + std::to_string(j) + " (chain): " + cudaGetErrorString(err));
        j += n_ops;
        continue;
      }
    }
    if (c.dry) {
      ++j;
      continue;
    }
    switch (o.type) {
      case SF_OP_GEMM: {
        const Tensor &A = g.T[o.in[0]], &B = g.T[o.in[1]], &C = g.T[o.out[0]];
        sfk::GemmArgs ga;
        ga.A = c.f(o.in[0]); ga.B = c.f(o.in[1]); ga.C = c.f(o.out[0]);
        ga.ta = o.flags & SF_GEMM_TA; ga.tb = o.flags & SF_GEMM_TB; ga.acc = o.flags & SF_GEMM_ACC;
        ga.M = C.rows; ga.N = C.cols; ga.K = ga.ta ? A.rows : A.cols;
        ga.lda = A.cols; ga.ldb = B.cols; ga.ldc = C.cols;
        ga.ws = c.b.ws; ga.counters = c.b.counters;
        ga.b_const = !g.op_written[o.in[1]];
        if (c.l2_keep) ga.l2_hint = c.l2_keep->count(o.in[1]) ? 1 : 2;
        {
          auto bk = c.b.blocked.find(o.in[1]);
          if (bk != c.b.blocked.end() && bk->second.second.ok && ga.M <= 8) {
            ga.Bblk = bk->second.first;
            ga.blk_qw = bk->second.second.qw;
            ga.blk_kper = bk->second.second.kper;
            ga.blk_cl = bk->second.second.cl;
          }
        }
        auto sa = c.b.shadow.find(o.in[0]);
        if (sa != c.b.shadow.end()) { ga.A = sa->second.first; ga.lda = sa->second.second; }
        auto sb = c.b.shadow.find(o.in[1]);
        if (sb != c.b.shadow.end()) { ga.B = sb->second.first; ga.ldb = sb->second.second; }
        auto pd = c.b.gemm_pad.find(j);
        if (pd != c.b.gemm_pad.end()) {
          const auto& pads = pd->second;
          const Tensor* xs[3] = {&A, &B, &C};
          const int ids[3] = {o.in[0], o.in[1], o.out[0]};
          for (int q = 0; q < 3; ++q) {
            if (!pads[q].p) continue;
            const Tensor& x = *xs[q];
            const bool load = q < 2 || ga.acc;  // C is read only when accumulating
            if (load) {
              err = sfk::launch_copy2d(c.ptr(ids[q]), static_cast<uint64_t>(x.cols) * 4, pads[q].p,
                                       static_cast<uint64_t>(pads[q].pitch) * 4, x.rows,
                                       static_cast<uint64_t>(x.cols) * 4, c.st);
              if (err != cudaSuccess) return fail(SF_ECUDA, std::string("pad: ") + cudaGetErrorString(err));
            }
          }
          if (pads[0].p) { ga.A = pads[0].p; ga.lda = pads[0].pitch; }
          if (pads[1].p) { ga.B = pads[1].p; ga.ldb = pads[1].pitch; ga.b_const = false; }
          if (pads[2].p) { ga.C = pads[2].p; ga.ldc = pads[2].pitch; }
          err = sfk::launch_gemm(ga, c.st);
          if (err == cudaSuccess && pads[2].p)
            err = sfk::launch_copy2d(pads[2].p, static_cast<uint64_t>(pads[2].pitch) * 4, c.ptr(o.out[0]),
                                     static_cast<uint64_t>(C.cols) * 4, C.rows,
                                     static_cast<uint64_t>(C.cols) * 4, c.st);
          break;
        }
        // Fuse a following BIAS_ACT into the GEMV epilogue when the GEMM output has no other
        // reader (same arithmetic order as the unfused pair, so results are bit-identical).
        if (j + 1 < e && !ga.acc && g.ops[j + 1].type == SF_OP_BIAS_ACT && g.ops[j + 1].in[0] == o.out[0] &&
            !(g.ops[j + 1].flags & SF_ACT_GELU) && C.kind != SF_OUTPUT &&
            (sfk::gemm_can_fuse_bias(ga.M, ga.N, ga.K, ga.ta, ga.tb, ga.ldb) || sfk::gemv_rows_eligible(ga))) {
          int readers = 0;
          for (const auto& q : g.ops)
            for (int t : op_reads(q)) readers += (t == o.out[0]);
          if (readers == 1) {
            const sf_op_desc& ba = g.ops[j + 1];
            ga.C = c.f(ba.out[0]);
            for (int i = 1; i < ba.n_in; ++i) ga.bias[i - 1] = c.f(ba.in[i]);
            ga.relu = ba.flags & SF_ACT_RELU;
            ga.ldc = g.T[ba.out[0]].cols;
            // ... and a following SOFTMAX of that output (the inference head) into the same
            // kernel: the last column block normalises the rows
            int used = 2;
            if (j + 2 < e && g.ops[j + 2].type == SF_OP_SOFTMAX && g.ops[j + 2].in[0] == ba.out[0] &&
                sfk::gemv_softmax_fusable(ga)) {
              ga.sm_out = c.f(g.ops[j + 2].out[0]);
              ga.sm_ldo = g.T[g.ops[j + 2].out[0]].cols;
              ga.sm_counter = c.b.counters + (g.counter_slots - 1);
              used = 3;
            }
            // the next GEMM of the chain streams constant weights: prefetch them to L2 from this
            // one (SF_GEMV_NEXT_PF=0 disables)
            static const bool next_pf = !(std::getenv("SF_GEMV_NEXT_PF") && std::getenv("SF_GEMV_NEXT_PF")[0] == '0');
            if (next_pf && !ga.Bblk && j + used < e && g.ops[j + used].type == SF_OP_GEMM) {
              const sf_op_desc& nx = g.ops[j + used];
              const Tensor& NB = g.T[nx.in[1]];
              if (!g.op_written[nx.in[1]] && !(nx.flags & (SF_GEMM_TA | SF_GEMM_TB)) && !c.b.shadow.count(nx.in[1])) {
                ga.pf_next = c.f(nx.in[1]);
                ga.pf_bytes = NB.nbytes;
              }
            }
            err = sfk::launch_gemm(ga, c.st);
            if (err != cudaSuccess) return fail(SF_ECUDA, "op " + std::to_string(j) + ": " + cudaGetErrorString(err));
            j += used;
            continue;
          }
        }
        err = sfk::launch_gemm(ga, c.st);
        break;
      }
      case SF_OP_BIAS_ACT: {
        const Tensor& z = g.T[o.in[0]];
        err = sfk::launch_bias_act(c.f(o.in[0]), c.f(o.in[1]), o.n_in > 2 ? c.f(o.in[2]) : nullptr,
                                   o.n_in > 3 ? c.f(o.in[3]) : nullptr, c.f(o.out[0]), z.rows, z.cols,
                                   (o.flags & SF_ACT_GELU) ? 2 : (o.flags & SF_ACT_RELU) ? 1 : 0, c.st,
                                   o.n_out > 1 ? c.f(o.out[1]) : nullptr);
        break;
      }
      case SF_OP_BIAS_ACT_BWD: {
        const Tensor& x = g.T[o.in[0]];
        err = sfk::launch_colsum(c.f(o.in[0]), c.f(o.in[1]), c.f(o.out[0]), c.f(o.out[1]), x.rows,
                                 x.cols, c.b.ws, c.b.counters, c.st, (o.flags & SF_ACT_GELU) ? 2 : 1);
        break;
      }
      case SF_OP_COLSUM: {
        const Tensor& x = g.T[o.in[0]];
        err = sfk::launch_colsum(c.f(o.in[0]), nullptr, nullptr, c.f(o.out[0]), x.rows, x.cols,
                                 c.b.ws, c.b.counters, c.st);
        break;
      }
      case SF_OP_SOFTMAX_CE: {
        const Tensor& l = g.T[o.in[0]];
        err = sfk::launch_softmax_ce(c.f(o.in[0]), reinterpret_cast<const int32_t*>(c.ptr(o.in[1])),
                                     c.f(o.out[0]), c.f(o.out[1]), l.rows, l.cols, c.b.ws,
                                     c.b.counters, c.st);
        break;
      }
      case SF_OP_SOFTMAX: {
        const Tensor& l = g.T[o.in[0]];
        err = sfk::launch_softmax(c.f(o.in[0]), c.f(o.out[0]), l.rows, l.cols, c.st);
        break;
      }
      case SF_OP_FEED: {
        const Tensor &pool = g.T[o.in[0]], &x = g.T[o.out[0]];
        err = sfk::launch_feed(c.ptr(o.in[0]), reinterpret_cast<const int32_t*>(c.ptr(o.in[1])),
                               c.ptr(o.out[0]), x.nbytes, pool.rows / x.rows, c.st);
        break;
      }
      case SF_OP_STEP_INC:
        err = sfk::launch_step_inc(reinterpret_cast<int32_t*>(c.ptr(o.out[0])), c.st);
        break;
      default:
        return fail(SF_EUNSUPPORTED, "op type");
    }
    if (err != cudaSuccess)
      return fail(SF_ECUDA, "op " + std::to_string(j) + ": " + cudaGetErrorString(err));
    ++j;
  }
  return SF_OK;
}

sf_status build_copy_list(Binding& b, const std::vector<sf_copy_desc>& descs, CopyList* out) {
  std::vector<sfk::DCopy> d;
  uint64_t chunks = 0, bytes = 0;
  for (const auto& s : descs) {
    sfk::DCopy x;
    x.src = static_cast<const uint8_t*>(s.src);
    x.dst = static_cast<uint8_t*>(s.dst);
    x.nbytes = s.nbytes;
    x.chunk_begin = chunks;
    chunks += s.span / 16;
    bytes += s.nbytes;
    d.push_back(x);
  }
  sfk::DCopy sent{};
  sent.chunk_begin = chunks;
  d.push_back(sent);
  void* dd;
  if (sf_status s = upload(b, d.data(), d.size() * sizeof(sfk::DCopy), &dd)) return s;
  out->d = static_cast<sfk::DCopy*>(dd);
  out->n = static_cast<int>(descs.size());
  out->total_chunks = chunks;
  out->bytes = bytes;
  return SF_OK;
}

sf_status build_peer_lists(sf_runtime* rt, Graph& g, Binding& src, Binding& dst) {
  SF_CK(cudaSetDevice(rt->slots[src.slot]->cuda));
  std::vector<CopyList> lists(g.parts.size());
  for (size_t k = 0; k < g.parts.size(); ++k) {
    std::vector<sf_copy_desc> ds;
    for (uint32_t t : g.live[k]) {
      const Tensor& x = g.T[t];
      ds.push_back({src.arena + x.offset, dst.arena + x.offset, x.nbytes, round_up(x.nbytes, 16)});
    }
    if (sf_status s = build_copy_list(src, ds, &lists[k])) return s;
  }
  src.peer[dst.slot] = std::move(lists);
  return SF_OK;
}

// ---------------------------------------------------------------------------------------
// Scheduler
// ---------------------------------------------------------------------------------------
Slot& slot_of(sf_runtime* rt, int s) { return *rt->slots[s]; }

sf_status ensure_events(sf_runtime* rt, Job& J) {
  if (!J.ev_sub.empty()) return SF_OK;
  const size_t n = rt->slots.size();
  J.ev_sub.assign(n, nullptr); J.ev_a.assign(n, nullptr); J.ev_b.assign(n, nullptr); J.ev_c.assign(n, nullptr);
  J.ev_r.assign(n, nullptr);
  J.ev_ring.assign(n * kEvRing, nullptr);
  J.ev_start.assign(n * kEvRing, nullptr);
  J.ev_ck.assign(n * kCkEvents, nullptr);
  int cur = 0;
  cudaGetDevice(&cur);
  for (size_t s = 0; s < n; ++s) {
    if (rt->slots[s]->remote) continue;
    SF_CK(cudaSetDevice(rt->slots[s]->cuda));
    SF_CK(cudaEventCreateWithFlags(&J.ev_sub[s], cudaEventDisableTiming));
    SF_CK(cudaEventCreate(&J.ev_r[s]));  // timing: device resume point
    for (int i = 0; i < kEvRing; ++i) {  // timing events: device intervals of subgraphs
      SF_CK(cudaEventCreate(&J.ev_ring[s * kEvRing + i]));
      SF_CK(cudaEventCreate(&J.ev_start[s * kEvRing + i]));
    }
    for (int i = 0; i < kCkEvents; ++i)
      SF_CK(cudaEventCreateWithFlags(&J.ev_ck[s * kCkEvents + i], cudaEventDisableTiming));
    SF_CK(cudaEventCreate(&J.ev_a[s]));
    SF_CK(cudaEventCreate(&J.ev_b[s]));
    SF_CK(cudaEventCreate(&J.ev_c[s]));
  }
  SF_CK(cudaSetDevice(cur));
  return SF_OK;
}

cudaError_t spin_event(cudaEvent_t ev) {
  for (;;) {
    cudaError_t e = cudaEventQuery(ev);
    if (e != cudaErrorNotReady) return e;
  }
}

// Millisecond-scale waits (host-tier D2H / H2D, peer stores) poll with short sleeps: a
// tight cudaEventQuery loop on this thread contends for the CUDA driver's locks with the
// dispatcher's kernel launches and stretches the preempter's launch chain.
// The first ~100 us are polled with short pauses: a sleep costs the OS timer slack (tens of
// us, often more), which dominated the preempt-to-resume of small live sets (C1: two relaxed
// waits per host round trip).
cudaError_t wait_event_relaxed(cudaEvent_t ev) {
  const uint64_t spin_until = now_ns() + 100000;
  for (;;) {
    cudaError_t e = cudaEventQuery(ev);
    if (e != cudaErrorNotReady) return e;
    if (now_ns() < spin_until) {
      for (int i = 0; i < 256; ++i) cpu_relax();
    } else {
      std::this_thread::sleep_for(std::chrono::microseconds(20));
    }
  }
}

float elapsed_us(cudaEvent_t a, cudaEvent_t b) {
  float ms = 0.f;
  if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) {
    cudaGetLastError();  // statistics only: never leave a stale error for the next launch
    return -1.f;
  }
  return ms * 1000.f;
}

// ---- stream memory operations (drain gate): driver entry points resolved at run time ----------
using StreamValueFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
StreamValueFn stream_mem_fn(const char* name) {
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &fn, cudaEnableDefault, &q) != cudaSuccess ||
      q != cudaDriverEntryPointSuccess)
    return nullptr;
  return reinterpret_cast<StreamValueFn>(fn);
}
StreamValueFn wait_value32() {
  static StreamValueFn f = stream_mem_fn("cuStreamWaitValue32");
  return f;
}
StreamValueFn write_value32() {
  static StreamValueFn f = stream_mem_fn("cuStreamWriteValue32");
  return f;
}
constexpr uint32_t kGateOpenAhead = 0x40000000u;  // G = next ticket + this: every ticket passes
void gate_open(Slot& S) {  // rt->m held
  S.gate[0] = S.next_ticket + kGateOpenAhead;
  std::atomic_thread_fence(std::memory_order_seq_cst);
  S.gate_held = false;
}

// ---- device clock (trace intervals on the GPU timeline, reading Q37) -------------
// One anchor: 3 stamp rounds on the slot's high-priority clock stream; the round with the
// tightest host window (launch .. value observed in pinned memory) becomes the anchor.
cudaError_t refresh_anchor(Slot& S) {
  cudaError_t e = cudaSetDevice(S.cuda);
  if (e != cudaSuccess) return e;
  Slot::Anchor best{nullptr, 0, 0, 0, ~0ull};
  for (int round = 0; round < 3; ++round) {
    volatile unsigned long long* h = S.clk_host;
    *h = 0ull;
    // E1 | stamp kernel (g = %globaltimer) | E2: the anchor is E1, whose GPU time is taken as
    // g - elapsed(E1, E2) / 2 (the stamp sits inside the bracket; a timing event recorded AFTER
    // the kernel can land tens of us late on a busy GPU)
    cudaEvent_t e1 = nullptr, e2 = nullptr;
    if ((e = cudaEventCreate(&e1)) != cudaSuccess) return e;
    if ((e = cudaEventCreate(&e2)) != cudaSuccess) { cudaEventDestroy(e1); return e; }
    const uint64_t h0 = now_ns();
    e = cudaEventRecord(e1, S.s_clk);
    if (e == cudaSuccess) e = sfk::launch_stamp(S.clk_dev, S.s_clk);
    if (e == cudaSuccess) e = cudaEventRecord(e2, S.s_clk);
    if (e != cudaSuccess) { cudaEventDestroy(e1); cudaEventDestroy(e2); return e; }
    unsigned long long g = 0;
    while ((g = *h) == 0ull) {
      if (now_ns() - h0 > 200000000ull) break;  // 200 ms: the device is saturated, skip
      cpu_relax();
    }
    const uint64_t h1 = now_ns();
    if ((e = cudaEventSynchronize(e2)) != cudaSuccess) { cudaEventDestroy(e1); cudaEventDestroy(e2); return e; }
    float br = 0.f;
    const bool ok = g != 0ull && cudaEventElapsedTime(&br, e1, e2) == cudaSuccess && br >= 0.f;
    cudaEventDestroy(e2);

    // round quality: the stamp's position inside its event bracket (br) is what the anchor's
    // GPU time rests on; the host side (h1 - g) has a ~0.2-1 us one-sided spread
    const uint64_t unc = static_cast<uint64_t>(static_cast<double>(br) * 1e6) + (h1 - h0) / 16;
    if (!ok || br > 0.02f || unc >= best.unc_ns) { cudaGetLastError(); cudaEventDestroy(e1); continue; }
    if (best.ev) cudaEventDestroy(best.ev);
    // the value was written at host time in [h0 + launch latency, h1 - write propagation]: the
    // launch side of that window is the long one, the write lands and is seen ~1 us after the
    // stamp, so h1 - 1 us is the host time of g
    const uint64_t g1 = g - static_cast<uint64_t>(static_cast<double>(br) * 0.5e6);
    best = Slot::Anchor{e1, h0, g1, static_cast<int64_t>(h1) - 700 - static_cast<int64_t>(g), unc};
  }
  if (!best.ev) return cudaSuccess;
  std::lock_guard<std::mutex> lk(S.clk_m);
  best.D = static_cast<double>(best.g_ns);
  if (!S.anchors.empty()) {
    float ms = 0.f;
    if (cudaEventElapsedTime(&ms, S.anchors.back().ev, best.ev) == cudaSuccess && ms >= 0.f)
      best.D = S.anchors.back().D + static_cast<double>(ms) * 1e6;
    else
      cudaGetLastError();
  }
  S.anchors.push_back(best);
  while (S.anchors.size() > 256) {
    cudaEventDestroy(S.anchors.front().ev);
    S.anchors.pop_front();
  }
  return cudaSuccess;
}

// CLOCK_MONOTONIC ns of a completed timing event of slot S enqueued at host time enq_ns (by the
// latest anchor enqueued at least 100 us earlier, so elapsed() is positive); 0 if unavailable.
uint64_t event_host_ns(Slot& S, cudaEvent_t ev, uint64_t enq_ns) {
  std::lock_guard<std::mutex> lk(S.clk_m);
  const Slot::Anchor* a = nullptr;
  for (auto it = S.anchors.rbegin(); it != S.anchors.rend(); ++it)
    if (it->enq_ns + 100000 <= enq_ns) { a = &*it; break; }
  if (!a) return 0;
  float ms = 0.f;
  if (cudaEventElapsedTime(&ms, a->ev, ev) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  // %globaltimer and CLOCK_MONOTONIC drift apart (~30 ppm measured on B200, scripts/
  // clock_probe.cu): the offset is interpolated between the anchors around the event (or
  // extrapolated along the last two), not held constant
  const double dev_ns = static_cast<double>(a->g_ns) + static_cast<double>(ms) * 1e6;
  const Slot::Anchor* b = nullptr;  // the next anchor after a, else the one before
  bool after = false;
  for (size_t i = 0; i < S.anchors.size(); ++i)
    if (&S.anchors[i] == a) {
      if (i + 1 < S.anchors.size()) { b = &S.anchors[i + 1]; after = true; }
      else if (i > 0) b = &S.anchors[i - 1];
      break;
    }
  double off = static_cast<double>(a->offset_ns);
  if (b && b->g_ns != a->g_ns) {
    const double slope = (static_cast<double>(b->offset_ns) - static_cast<double>(a->offset_ns)) /
                         (static_cast<double>(b->g_ns) - static_cast<double>(a->g_ns));
    if (std::fabs(slope) < 1e-3) off += slope * (dev_ns - static_cast<double>(a->g_ns));
    (void)after;
  }
  return static_cast<uint64_t>(dev_ns + off);
}

// Device-timeline position D of a completed timing event (see Slot::Anchor::D), by the latest
// anchor enqueued at least 100 us before it; NaN if unavailable.
double event_dev_D(Slot& S, cudaEvent_t ev, uint64_t enq_ns) {
  std::lock_guard<std::mutex> lk(S.clk_m);
  const Slot::Anchor* a = nullptr;
  for (auto it = S.anchors.rbegin(); it != S.anchors.rend(); ++it)
    if (it->enq_ns + 100000 <= enq_ns) { a = &*it; break; }
  if (!a) return std::nan("");
  float ms = 0.f;
  if (cudaEventElapsedTime(&ms, a->ev, ev) != cudaSuccess) {
    cudaGetLastError();
    return std::nan("");
  }
  return a->D + static_cast<double>(ms) * 1e6;
}

// CLOCK_MONOTONIC ns of device-timeline position D with the slot's CURRENT anchors: the
// offset host - D, known at every anchor, is interpolated linearly in D between the anchors
// around it (held at the ends).  One mapping for all trace events read together, so it is
// monotone in D: the device order of events survives into the trace.
uint64_t dev_D_to_host(Slot& S, double D) {
  std::lock_guard<std::mutex> lk(S.clk_m);
  if (S.anchors.empty() || std::isnan(D)) return 0;
  auto off = [](const Slot::Anchor& a) {
    return static_cast<double>(a.g_ns) + static_cast<double>(a.offset_ns) - a.D;
  };
  const auto& A = S.anchors;
  size_t hi = 0;
  while (hi < A.size() && A[hi].D <= D) ++hi;
  double o;
  if (hi == 0) o = off(A.front());
  else if (hi == A.size()) o = off(A.back());
  else {
    const Slot::Anchor &a = A[hi - 1], &b = A[hi];
    const double w = b.D > a.D ? (D - a.D) / (b.D - a.D) : 0.0;
    o = off(a) + w * (off(b) - off(a));
  }
  return static_cast<uint64_t>(D + o);
}

void clock_main(sf_runtime* rt);

// Inference GEMV weights (M <= 8, constant B): blocked copies allocated at bind (reading Q39).
sf_status alloc_blocked(Graph& g, Binding& b) {
  static const bool on = !(std::getenv("SF_GEMV_BLOCKED") && std::getenv("SF_GEMV_BLOCKED")[0] == '0');
  if (!on) return SF_OK;
  for (const auto& o : g.ops) {
    if (o.type != SF_OP_GEMM || (o.flags & (SF_GEMM_TA | SF_GEMM_TB | SF_GEMM_ACC)) || g.op_written[o.in[1]])
      continue;
    const Tensor &Bt = g.T[o.in[1]], &Ct = g.T[o.out[0]];
    if (Ct.rows > 8 || b.shadow.count(o.in[1]) || b.blocked.count(o.in[1])) continue;
    const sfk::GemvBlockPlan pl = sfk::plan_gemv_block(Ct.rows, Bt.cols, Bt.rows);
    if (!pl.ok) continue;
    void* d = nullptr;
    SF_CK(cudaMalloc(&d, pl.bytes));
    b.dev_allocs.push_back(d);
    b.blocked[o.in[1]] = {d, pl};
  }
  return SF_OK;
}
// SF_INFER_GRAPH: 0 direct launches only; 1 every request through the captured graph; 2
// (default, reading Q36) the graph only for requests that find the device free (a
// preempting request's kernels are enqueued behind the drain event directly, which starts them
// sooner; a request landing during a host round trip gets one launch call and one command fetch
// over the busy PCIe link instead of three)
int infer_graph_mode() {
  static const int m = std::getenv("SF_INFER_GRAPH") ? std::atoi(std::getenv("SF_INFER_GRAPH")) : 2;
  return m;
}

sf_status launch_subgraph_ops(Capture& c, int k);

// Captures the request chain of an inference binding once: copy(in -> arena input), the
// subgraph kernels (programmatic dependent launch as on the direct path), copy(arena output ->
// out).  The two copy nodes are found by their kernel and patched per request.
void build_req_graph(Graph& g, Binding& B, bool pdl) {
  Binding::ReqGraph& R = B.rg;
  if (R.state != 0) return;
  R.state = -1;
  if (g.input_tid < 0 || g.output_tid < 0) return;
  const Tensor &tin = g.T[g.input_tid], &tout = g.T[g.output_tid];
  if (tin.nbytes % 4 || tout.nbytes % 4) return;
  cudaStream_t st = nullptr;
  if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess) { cudaGetLastError(); return; }
  const bool pdl_was = sfk::pdl_enabled();
  sfk::set_pdl(pdl);
  const uint64_t l0 = sfk::launches();
  bool ok = cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal) == cudaSuccess;
  cudaGraph_t graph = nullptr;
  if (ok) {
    uint8_t* ain = B.arena + tin.offset;
    uint8_t* aout = B.arena + tout.offset;
    ok = sfk::launch_copy(ain, ain, tin.nbytes, st) == cudaSuccess;  // src patched per request
    for (size_t k = 0; ok && k < B.versions.size(); ++k) {
      Capture c{g, B, st, false, &B.prepared};
      ok = launch_subgraph_ops(c, static_cast<int>(k)) == SF_OK;
    }
    ok = ok && sfk::launch_copy(aout, aout, tout.nbytes, st) == cudaSuccess;  // dst patched
    const cudaError_t e = cudaStreamEndCapture(st, &graph);
    ok = ok && e == cudaSuccess && graph;
  }
  const uint64_t nk = sfk::launches() - l0;
  sfk::count_launch(uint64_t(0) - nk);  // captured, not launched: counted at each replay
  sfk::set_pdl(pdl_was);
  cudaStreamDestroy(st);
  if (!ok) {
    cudaGetLastError();
    if (graph) cudaGraphDestroy(graph);
    return;
  }
  size_t n = 0;
  cudaGraphGetNodes(graph, nullptr, &n);
  std::vector<cudaGraphNode_t> nodes(n);
  cudaGraphGetNodes(graph, nodes.data(), &n);
  for (auto nd : nodes) {
    cudaGraphNodeType t;
    if (cudaGraphNodeGetType(nd, &t) != cudaSuccess || t != cudaGraphNodeTypeKernel) continue;
    cudaKernelNodeParams kp{};
    if (cudaGraphKernelNodeGetParams(nd, &kp) != cudaSuccess || kp.func != sfk::copy_kernel_fn()) continue;
    size_t ndep = 0, nout = 0;
    cudaGraphNodeGetDependencies(nd, nullptr, &ndep);
    cudaGraphNodeGetDependentNodes(nd, nullptr, &nout);
    if (ndep == 0) { R.in_node = nd; R.in_grid = kp.gridDim; R.in_block = kp.blockDim; }
    else if (nout == 0) { R.out_node = nd; R.out_grid = kp.gridDim; R.out_block = kp.blockDim; }
  }
  cudaGraphExec_t exec = nullptr;
  if (!R.in_node || !R.out_node || cudaGraphInstantiate(&exec, graph, 0) != cudaSuccess) {
    cudaGetLastError();
    cudaGraphDestroy(graph);
    R.in_node = R.out_node = nullptr;
    return;
  }
  R.graph = graph;
  R.exec = exec;
  R.kernels = nk;
  R.state = 1;
}

// Patches the request's buffers into the captured chain and launches it (one API call).
cudaError_t launch_req_graph(Binding& B, const Tensor& tin, const Tensor& tout, const void* in, void* out,
                             cudaStream_t st) {
  Binding::ReqGraph& R = B.rg;
  const uint8_t* src_in = static_cast<const uint8_t*>(in);
  uint8_t* dst_in = B.arena + tin.offset;
  uint64_t n_in = tin.nbytes;
  void* a_in[] = {&src_in, &dst_in, &n_in};
  cudaKernelNodeParams kp{};
  kp.func = const_cast<void*>(sfk::copy_kernel_fn());
  kp.gridDim = R.in_grid;
  kp.blockDim = R.in_block;
  kp.kernelParams = a_in;
  cudaError_t e = cudaGraphExecKernelNodeSetParams(R.exec, R.in_node, &kp);
  const uint8_t* src_out = B.arena + tout.offset;
  uint8_t* dst_out = static_cast<uint8_t*>(out);
  uint64_t n_out = tout.nbytes;
  void* a_out[] = {&src_out, &dst_out, &n_out};
  kp.gridDim = R.out_grid;
  kp.blockDim = R.out_block;
  kp.kernelParams = a_out;
  if (e == cudaSuccess) e = cudaGraphExecKernelNodeSetParams(R.exec, R.out_node, &kp);
  if (e == cudaSuccess) e = cudaGraphLaunch(R.exec, st);
  if (e == cudaSuccess) sfk::count_launch(R.kernels);
  return e;
}

// Lay the current weights out into the blocked copies (stream-ordered on st).
void layout_blocked(const Graph& g, Binding& b, cudaStream_t st) {
  for (auto& [t, d] : b.folded) {
    const Tensor& Wt = g.T[t];
    if (sfk::launch_chain_w0t_layout(reinterpret_cast<const float*>(b.arena + Wt.offset), Wt.cols, Wt.rows,
                                     Wt.cols, d, st) != cudaSuccess)
      cudaGetLastError();
  }
  for (auto& [t, e] : b.blocked) {
    const Tensor& Bt = g.T[t];
    if (sfk::launch_gemv_block_layout(reinterpret_cast<const float*>(b.arena + Bt.offset), e.first, Bt.rows,
                                      Bt.cols, Bt.cols, e.second, st) != cudaSuccess) {
      cudaGetLastError();
      e.second.ok = false;
    }
  }
}

bool slot_has_inference(sf_runtime* rt, int s) { return !slot_of(rt, s).q.empty(); }

// A training job of priority > min_prio (>= when or_equal) is present on slot s: running or
// waiting for the device there, or parked from s on the host tier (it swaps back into s).
// Jobs moving to a peer, explicitly parked (sf_preempt) or finished are not present.
const Job* present_job(sf_runtime* rt, int s, const Job* me, int min_prio, bool or_equal) {
  for (const auto& Jp : rt->jobs) {
    const Job& o = *Jp;
    if (&o == me || o.dev != s) continue;
    const int p = o.g->priority;
    if (or_equal ? p < min_prio : p <= min_prio) continue;
    if (o.state == SF_JOB_RUNNING || o.state == SF_JOB_STOPPING ||
        (o.state == SF_JOB_MIGRATING && o.preempt_target == SF_TARGET_HOST))
      return &o;
  }
  return nullptr;
}
// Higher-priority training on J's slot (the Fig. 7 preempter).
const Job* higher_training(sf_runtime* rt, const Job& J, int s) {
  return present_job(rt, s, &J, J.g->priority, false);
}

// Device-side kernel duration stamps (globaltimer): reset {start, end} = {~0, 0}.
cudaError_t tstamp_reset(unsigned long long* t, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(t, 0xFF, sizeof(unsigned long long), st);
  return e == cudaSuccess ? cudaMemsetAsync(t + 1, 0, sizeof(unsigned long long), st) : e;
}
double tstamp_us(const unsigned long long* t) {  // after the stream completed
  unsigned long long h[2] = {0, 0};
  if (cudaMemcpy(h, t, sizeof(h), cudaMemcpyDeviceToHost) != cudaSuccess) {
    cudaGetLastError();
    return -1.0;
  }
  if (h[1] < h[0]) return -1.0;
  return (h[1] - h[0]) * 1e-3;
}

// Poison the non-DATASET tensors of a released arena (test mode): a missing live tensor
// then reads as NaN / -1 after resume.
cudaError_t poison(Binding& b, cudaStream_t st) {
  for (auto [off, len] : b.poison_ranges) {
    cudaError_t e = sfk::launch_fill(b.arena + off, len, 0xFF, st);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}


// Copy-engine transfers.  A segment list is issued in ~2 MB batches (large segments split),
// one cudaMemcpyAsync per segment (the batched copy API is closed on this GPU pool: it raised
// Xid faults), so no SM runs for the copy.  With `yield`, at most two batches are in flight
// and none is issued while a request is queued or running on the slot: copy-engine traffic
// over PCIe slows a concurrent batch-1 forward by ~45% on B200 (scripts/infer_bench.py
// COPY=d2h: 50 -> 74 us; reading Q22).  Returns once every batch has been issued and (yield)
// has completed.
struct Seg {
  void* dst;
  const void* src;
  size_t n;
};

cudaError_t issue_batch(std::vector<void*>& d, std::vector<void*>& s, std::vector<size_t>& n,
                        cudaStream_t st) {
  for (size_t i = 0; i < d.size(); ++i) {
    const cudaError_t e = cudaMemcpyAsync(d[i], s[i], n[i], cudaMemcpyDefault, st);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

cudaError_t ce_segments(Job& J, Slot& S, int slot, const std::vector<Seg>& segs, cudaStream_t st,
                        bool yield) {
  constexpr size_t kChunk = size_t(2) << 20;
  size_t si = 0, so = 0;  // cursor: segment, offset inside it
  int head = 0, n_inflight = 0;  // ring of 2 events
  std::vector<void*> bd, bs;
  std::vector<size_t> bn;
  auto busy = [&] {
    const int o = S.owner.load(std::memory_order_acquire);
    return S.qn.load(std::memory_order_acquire) > 0 || o == kInferOwner;
  };
  while (si < segs.size() || n_inflight > 0) {
    if (si < segs.size() && (!yield || (n_inflight < 2 && !busy()))) {
      bd.clear(); bs.clear(); bn.clear();
      size_t got = 0;
      while (si < segs.size() && got < kChunk) {
        const Seg& g = segs[si];
        const size_t n = std::min(kChunk - got, g.n - so);
        if (n > 0) {
          bd.push_back(static_cast<uint8_t*>(g.dst) + so);
          bs.push_back(const_cast<uint8_t*>(static_cast<const uint8_t*>(g.src) + so));
          bn.push_back(n);
        }
        got += n;
        so += n;
        if (so == g.n) { ++si; so = 0; }
      }
      cudaError_t e = issue_batch(bd, bs, bn, st);
      if (e == cudaSuccess && yield) e = cudaEventRecord(J.ev_ck[slot * kCkEvents + (head + n_inflight) % 2], st);
      if (e != cudaSuccess) return e;
      if (yield) ++n_inflight;
      continue;
    }
    if (n_inflight > 0) {
      const cudaError_t q = cudaEventQuery(J.ev_ck[slot * kCkEvents + head]);
      if (q == cudaSuccess) {
        head = (head + 1) % 2;
        --n_inflight;
        continue;
      }
      if (q != cudaErrorNotReady) return q;
    }
    for (int i = 0; i < 64; ++i) cpu_relax();
  }
  return cudaSuccess;
}

cudaError_t yielding_copy(Job& J, Slot& S, int slot, void* dst, const void* src, size_t bytes,
                          cudaStream_t st) {
  return ce_segments(J, S, slot, {Seg{dst, src, bytes}}, st, true);
}

// Full-duplex host round trip (cfg.host_duplex): when nothing waits for the device at the
// park, the job need not stay parked, so each 2 MB chunk of the packed staging goes D2H on the
// migration stream and comes back H2D on the training stream as soon as it landed in pinned
// memory (a stream-ordered event wait, no host sync).  Both PCIe directions then run at once
// and the round trip costs max(S/d2h, S/h2d) instead of S/d2h + S/h2d.  With `poison_chunks`
// each device staging chunk is filled with 0xFF between its D2H and its H2D, so a chunk that
// does not come back from pinned memory shows up in the unpacked state.  Yields like
// ce_segments: at most two chunks in flight per direction, none issued while a request is
// queued or running on the slot.  Returns once every chunk is back in device staging.
cudaError_t duplex_round_trip(Job& J, Slot& S, int slot, uint8_t* dstg, uint8_t* hstg, size_t total,
                              bool poison_chunks) {
  static const size_t kChunk = std::getenv("SF_DUPLEX_CHUNK_KB")
                                   ? size_t(std::atoi(std::getenv("SF_DUPLEX_CHUNK_KB"))) << 10
                                   : size_t(2) << 20;
  static const size_t kDepth = std::getenv("SF_DUPLEX_DEPTH")
                                   ? size_t(std::max(1, std::min(2, std::atoi(std::getenv("SF_DUPLEX_DEPTH")))))
                                   : 2;
  // D2H traffic delays a concurrent request's command / completion traffic the most
  // (reading Q34): SF_DUPLEX_DEPTH_D2H caps the D2H chunks in flight separately
  static const size_t kDepthD2H = std::getenv("SF_DUPLEX_DEPTH_D2H")
                                      ? size_t(std::max(1, std::min(2, std::atoi(std::getenv("SF_DUPLEX_DEPTH_D2H")))))
                                      : kDepth;
  constexpr int R = 4;  // event ring per direction (kCkEvents / 2)
  // small live sets (2-8 MB): R equal chunks all issued at once (D2H on the migration stream,
  // each H2D waiting on its chunk's event on the device), so the two directions overlap without
  // host round trips between chunks.  At most one chunk of 2 MB (C1's 1.6-2.4 MB): one D2H then
  // one H2D — measured cheaper than any split at that size, where every extra copy costs more
  // in fixed latency than the overlap saves (scripts/pcie_small.py: 1.6 MB D2H 34 us, H2D 35,
  // both 71 us back to back, 95-272 us as 2-8 overlapped chunks)
  const bool upfront = !std::getenv("SF_DUPLEX_CHUNK_KB") && total > kChunk && total <= R * kChunk;
  const size_t chunk = upfront ? std::max<size_t>(size_t(64) << 10, ((total + R - 1) / R + 4095) / 4096 * 4096)
                               : kChunk;
  const size_t depth = upfront ? R : kDepth, depth_d2h = upfront ? R : kDepthD2H;
  const size_t nch = (total + chunk - 1) / chunk;
  size_t nd = 0, nh = 0, cd = 0, ch = 0;  // D2H / H2D issued, D2H / H2D completed
  cudaEvent_t* evd = &J.ev_ck[slot * kCkEvents];
  cudaEvent_t* evh = evd + R;
  auto busy = [&] {
    const int o = S.owner.load(std::memory_order_acquire);
    return S.qn.load(std::memory_order_acquire) > 0 || o == kInferOwner;
  };
  static const bool quiet = !(std::getenv("SF_DUPLEX_QUIET") && std::getenv("SF_DUPLEX_QUIET")[0] == '0');
  // SF_DUPLEX_HOSTORDER=1: issue H2D(c) once the host saw D2H(c) complete (no cross-engine
  // event wait on the device)
  static const bool host_order = std::getenv("SF_DUPLEX_HOSTORDER") && std::getenv("SF_DUPLEX_HOSTORDER")[0] == '1';
  while (ch < nch) {
    bool progressed = false;
    if (quiet && busy()) {
      // a request is queued or running: no CUDA calls from this thread (driver-lock
      // contention stretches the dispatcher's launch chain); in-flight chunks drain alone
      std::this_thread::sleep_for(std::chrono::microseconds(10));
      continue;
    }
    if (!busy()) {
      if (nd < nch && nd - cd < depth_d2h && nd - nh < static_cast<size_t>(R)) {
        const size_t off = nd * chunk, n = std::min(chunk, total - off);
        cudaError_t e = cudaMemcpyAsync(hstg + off, dstg + off, n, cudaMemcpyDeviceToHost, S.s_mig);
        if (e == cudaSuccess && poison_chunks) e = sfk::launch_fill(dstg + off, n, 0xFF, S.s_mig);
        if (e == cudaSuccess) e = cudaEventRecord(evd[nd % R], S.s_mig);
        if (e != cudaSuccess) return e;
        ++nd;
        progressed = true;
      }
      if (nh < (host_order ? cd : nd) && nh - ch < depth) {
        const size_t off = nh * chunk, n = std::min(chunk, total - off);
        cudaError_t e = host_order ? cudaSuccess : cudaStreamWaitEvent(S.s_train, evd[nh % R], 0);
        if (e == cudaSuccess) e = cudaMemcpyAsync(dstg + off, hstg + off, n, cudaMemcpyHostToDevice, S.s_train);
        if (e == cudaSuccess) e = cudaEventRecord(evh[nh % R], S.s_train);
        if (e != cudaSuccess) return e;
        ++nh;
        progressed = true;
      }
    }
    if (cd < nd) {
      const cudaError_t q = cudaEventQuery(evd[cd % R]);
      if (q == cudaSuccess) { ++cd; progressed = true; }
      else if (q != cudaErrorNotReady) return q;
    }
    if (ch < nh) {
      const cudaError_t q = cudaEventQuery(evh[ch % R]);
      if (q == cudaSuccess) { ++ch; progressed = true; }
      else if (q != cudaErrorNotReady) return q;
    }
    if (!progressed) for (int i = 0; i < 64; ++i) cpu_relax();
  }
  return cudaSuccess;
}

// Copy-engine-only migration (SF_MIG_CE): the per-tensor segments of cut k.
//   to_host: arena -> pinned staging payloads; from_host: staging payloads -> arena;
//   peer: arena -> peer arena (same offsets).
std::vector<Seg> cut_segments(const Graph& g, int k, uint8_t* arena, uint8_t* other, int dir) {
  std::vector<Seg> v;
  v.reserve(g.live[k].size());
  for (size_t e = 0; e < g.live[k].size(); ++e) {
    const Tensor& t = g.T[g.live[k][e]];
    if (dir == 0) v.push_back({other + g.payload_off[k][e], arena + t.offset, t.nbytes});
    else if (dir == 1) v.push_back({arena + t.offset, other + g.payload_off[k][e], t.nbytes});
    else v.push_back({other + t.offset, arena + t.offset, t.nbytes});
  }
  return v;
}

// The staging header of cut k (iter patched) and zero padding, written by the CPU straight
// into pinned staging (the copy engines write only the payloads): byte-identical to a pack.
void write_host_header(const Graph& g, int k, int64_t iter, uint8_t* stg) {
  std::memcpy(stg, g.header[k].data(), g.header[k].size());
  std::memcpy(stg + 16, &iter, sizeof(iter));
  const auto& off = g.payload_off[k];
  for (size_t e = 0; e < off.size(); ++e) {
    const uint64_t end = off[e] + g.T[g.live[k][e]].nbytes;
    const uint64_t next = e + 1 < off.size() ? off[e + 1] : g.staging_total[k];
    if (next > end) std::memset(stg + end, 0, next - end);
  }
}

// Host-tier swap-in unpack grid in waves (SF_UNPACK_WAVES, default 1): short-lived CTAs let a
// request that arrives during the unpack get SMs after one wave instead of after the walk.
int unpack_waves() {
  static const int w = std::getenv("SF_UNPACK_WAVES") ? std::max(1, std::atoi(std::getenv("SF_UNPACK_WAVES"))) : 1;
  return w;
}

// Preempt J at its current boundary (rt->m held on entry and on return).
sf_status do_preempt(sf_runtime* rt, Job& J, std::unique_lock<std::mutex>& lk) {
  Graph& g = *J.g;
  const bool expl = J.preempt_park;  // explicit sf_preempt: park until sf_resume
  const int target = J.preempt_target;
  const int src = J.dev;
  const int k = J.k;
  J.preempt_req = false;
  J.state = SF_JOB_MIGRATING;
  J.last_stop = now_ns();
  J.cut = sf_cut_info{};
  J.cut.iter = J.it;
  J.cut.k = k;
  J.cut.n_tensors = static_cast<int32_t>(g.live[k].size());
  J.cut.live_bytes = g.live_bytes[k];
  J.cut.t_req_ns = J.t_req;
  J.cut.t_stop_ns = J.last_stop;
  J.cut.src_dev = src;
  J.cut.dst_dev = target;
  J.cut_ready = true;
  J.mig_enqueued = false;
  for (Request* r : slot_of(rt, src).q)
    if (r->preempted_job < 0) {
      r->preempted_job = static_cast<int>(J.id);
      r->cut_iter = J.it;
      r->cut_k = k;
    }
  rt->cv.notify_all();
  Slot& S = slot_of(rt, src);
  Binding& B = *g.bind[src];
  if (rt->cfg.defer_migration) {
    // the preempter runs first with the whole device; the copy starts once it drained
    rt->cv.wait(lk, [&] {
      return rt->shutting_down || (!slot_has_inference(rt, src) && S.owner != kInferOwner);
    });
  }
  lk.unlock();

  auto cuda_fail = [&](cudaError_t e, const char* what) {
    lk.lock();
    J.error = std::string(what) + ": " + cudaGetErrorString(e);
    J.state = SF_JOB_FAILED;
    rt->cv.notify_all();
    return fail(SF_ECUDA, J.error);
  };
  cudaError_t e;
  // The migration stream reads the arena only after everything already enqueued on the
  // training stream (a pending swap-in or stream-ordered peer arrival) has landed.
  if ((e = cudaSetDevice(S.cuda)) != cudaSuccess) return cuda_fail(e, "set device");
  if ((e = cudaEventRecord(J.ev_sub[src], S.s_train)) != cudaSuccess ||
      (e = cudaStreamWaitEvent(S.s_mig, J.ev_sub[src], 0)) != cudaSuccess)
    return cuda_fail(e, "order migration after training stream");
  // Re-preempted before running anything since its swap-in from this slot's pinned
  // staging: that copy of L_k is still current, so park again without pack + D2H.
  const bool repark = target == SF_TARGET_HOST && J.stamp_resume && J.parked_slot == src &&
                      J.parked_iter == J.it && J.parked_k == k;
  if (target == SF_TARGET_HOST) {
    // ---- host tier: pack (+ D2H), park, swap back in ------------------------------
    // SF_MIG_CE: no pack kernel; the CPU writes the header, the copy engines the payloads
    const bool ce = rt->cfg.migration_engine == SF_MIG_CE;
    const bool zc = !ce && (rt->cfg.host_mode == SF_HOST_ZC || B.staging == nullptr);
    tstamp_reset(S.tstamp, S.s_mig);
    cudaEventRecord(J.ev_a[src], S.s_mig);
    if (repark) {
      cudaEventRecord(J.ev_b[src], S.s_mig);
      e = cudaSuccess;
    } else if (ce) {
      write_host_header(g, k, J.it, B.host_staging);
      cudaEventRecord(J.ev_b[src], S.s_mig);
      e = cudaSuccess;
    } else if (zc) {
      const CopyList& L = B.pack_zc[k];
      e = sfk::launch_mtcopy(L.d, L.n, L.total_chunks, J.it, S.s_mig, S.tstamp);
      cudaEventRecord(J.ev_b[src], S.s_mig);
    } else {
      const CopyList& L = B.pack[k];
      e = sfk::launch_mtcopy(L.d, L.n, L.total_chunks, J.it, S.s_mig, S.tstamp);
      cudaEventRecord(J.ev_b[src], S.s_mig);
    }
    if (e != cudaSuccess) return cuda_fail(e, "pack");
    lk.lock();
    J.mig_enqueued = true;
    rt->cv.notify_all();
    // nothing waits for the device (its queue drained, no higher-priority job present): the
    // swap-in may start at once, chunk by chunk, while the rest is still going out
    const bool duplex = rt->cfg.host_duplex && !expl && !repark && !ce && !zc && B.staging &&
                        !slot_has_inference(rt, src) && S.owner != kInferOwner &&
                        !higher_training(rt, J, src);
    lk.unlock();
    if (duplex) {
      if ((e = duplex_round_trip(J, S, src, B.staging, B.host_staging, g.staging_total[k],
                                 rt->cfg.poison_released != 0)) != cudaSuccess)
        return cuda_fail(e, "duplex D2H/H2D");
      if (rt->cfg.poison_released) {  // the released arena, before the unpack reads staging
        if ((e = poison(B, S.s_mig)) != cudaSuccess) return cuda_fail(e, "poison");
      }
      cudaEventRecord(J.ev_sub[src], S.s_mig);
      cudaStreamWaitEvent(S.s_train, J.ev_sub[src], 0);
      cudaEventRecord(J.ev_c[src], S.s_train);  // round trip complete
    } else {
      if (!repark && !zc &&
          (e = ce ? ce_segments(J, S, src, cut_segments(g, k, B.arena, B.host_staging, 0), S.s_mig, true)
                  : yielding_copy(J, S, src, B.host_staging, B.staging, g.staging_total[k], S.s_mig)) !=
              cudaSuccess)
        return cuda_fail(e, "D2H");
      cudaEventRecord(J.ev_c[src], S.s_mig);
    }
    if ((e = wait_event_relaxed(J.ev_c[src])) != cudaSuccess) return cuda_fail(e, "pack wait");
    float pack_us = repark || ce ? 0.f : static_cast<float>(tstamp_us(S.tstamp));  // kernel-only duration
    if (pack_us < 0.f) pack_us = elapsed_us(J.ev_a[src], J.ev_b[src]);
    // duplex: the whole round trip (both directions overlapped), else the D2H alone
    const float d2h_us = repark ? 0.f : elapsed_us(J.ev_b[src], J.ev_c[src]);
    if (rt->cfg.poison_released && !duplex) {
      if ((e = poison(B, S.s_mig)) != cudaSuccess) return cuda_fail(e, "poison");
      if ((e = cudaStreamSynchronize(S.s_mig)) != cudaSuccess) return cuda_fail(e, "poison sync");
    }
    lk.lock();
    J.pack_us = pack_us;
    J.xfer_us = d2h_us;
    J.parked_slot = src;
    J.parked_iter = J.it;
    J.parked_k = k;
    J.n_repark += repark ? 1 : 0;
    int dst = src;
    if (expl) {
      J.state = SF_JOB_PREEMPTED;
      rt->cv.notify_all();
      rt->cv.wait(lk, [&] { return J.resume_req || J.stop_req || rt->shutting_down; });
      if (!J.resume_req) { J.state = SF_JOB_DONE; rt->cv.notify_all(); return SF_OK; }
      dst = J.resume_dev;
      J.resume_req = false;
    } else if (!duplex) {
      // swap back in once the device's inference queue drained (reading Q4/Q13) and no
      // higher-priority training job is present on it
      rt->cv.wait(lk, [&] {
        return rt->shutting_down || (!slot_has_inference(rt, src) && S.owner != kInferOwner &&
                                     !higher_training(rt, J, src));
      });
    }
    Slot& D = slot_of(rt, dst);
    Binding& BD = *g.bind[dst];
    lk.unlock();
    if ((e = cudaSetDevice(D.cuda)) != cudaSuccess) return cuda_fail(e, "set device");
    if (dst != src) {  // as for the peer store: dst's arena may still be being released (poison)
      cudaEventRecord(J.ev_sub[dst], D.s_mig);
      cudaStreamWaitEvent(D.s_train, J.ev_sub[dst], 0);
    }
    cudaEventRecord(J.ev_a[dst], D.s_train);
    // the parked bytes live in the source binding's pinned staging; a ZC swap-in reads
    // them in place when resuming on the same slot, otherwise H2D + unpack
    tstamp_reset(D.tstamp + 2, D.s_train);
    if (duplex) {  // the H2D already ran (its time is in xfer_us): unpack only
      cudaEventRecord(J.ev_b[dst], D.s_train);
      const CopyList& L = BD.unpack[k];
      e = sfk::launch_mtcopy(L.d, L.n, L.total_chunks, -1, D.s_train, D.tstamp + 2, unpack_waves());
    } else if (ce) {
      e = ce_segments(J, D, dst, cut_segments(g, k, BD.arena, B.host_staging, 1), D.s_train, true);
      cudaEventRecord(J.ev_b[dst], D.s_train);
    } else if (zc && dst == src) {
      const CopyList& L = BD.unpack_zc[k];
      e = sfk::launch_mtcopy(L.d, L.n, L.total_chunks, -1, D.s_train, D.tstamp + 2);
      cudaEventRecord(J.ev_b[dst], D.s_train);
    } else if (!BD.staging) {
      e = cudaErrorInvalidValue;
    } else {
      e = yielding_copy(J, D, dst, BD.staging, B.host_staging, g.staging_total[k], D.s_train);
      cudaEventRecord(J.ev_b[dst], D.s_train);
      if (e == cudaSuccess) {
        const CopyList& L = BD.unpack[k];
        e = sfk::launch_mtcopy(L.d, L.n, L.total_chunks, -1, D.s_train, D.tstamp + 2, unpack_waves());
      }
    }
    if (e != cudaSuccess) return cuda_fail(e, "unpack");
    cudaEventRecord(J.ev_c[dst], D.s_train);
    // Hold no device token while the swap-in lands: a request arriving during the H2D runs
    // at once instead of queueing behind a resumed subgraph that waits for the copy; the
    // driver then re-parks (no copy: nothing ran) if requests are pending.
    if ((e = wait_event_relaxed(J.ev_c[dst])) != cudaSuccess) return cuda_fail(e, "swap-in wait");
    lk.lock();
    J.dev = dst;
  } else {
    // ---- peer tier: fused peer store into the target's arena over NVLink -----------
    J.parked_slot = -1;
    auto it = B.peer.find(target);
    if (it == B.peer.end()) {
      lk.lock();
      J.state = SF_JOB_FAILED;
      J.error = "no peer list to target slot";
      rt->cv.notify_all();
      return fail(SF_EINVAL, J.error);
    }
    const CopyList& L = it->second[k];
    {
      // the target arena was released by an earlier move out of that slot, whose clean-up
      // (the poison fill in test mode) runs on the TARGET slot's migration stream: the store
      // into it waits for that stream (a remote slot synchronised its own before the handoff)
      Slot& T0 = slot_of(rt, target);
      if (!T0.remote) {
        if ((e = cudaSetDevice(T0.cuda)) != cudaSuccess ||
            (e = cudaEventRecord(J.ev_sub[target], T0.s_mig)) != cudaSuccess ||
            (e = cudaSetDevice(S.cuda)) != cudaSuccess ||
            (e = cudaStreamWaitEvent(S.s_mig, J.ev_sub[target], 0)) != cudaSuccess)
          return cuda_fail(e, "order peer store after the target's migration stream");
      }
    }
    tstamp_reset(S.tstamp, S.s_mig);
    cudaEventRecord(J.ev_a[src], S.s_mig);
    if (rt->cfg.migration_engine == SF_MIG_CE)  // copy engines over NVLink, no SM work
      e = ce_segments(J, S, src, cut_segments(g, k, B.arena, g.bind[target]->arena, 2), S.s_mig, false);
    else
      e = sfk::launch_mtcopy(L.d, L.n, L.total_chunks, -1, S.s_mig, S.tstamp);
    if (e != cudaSuccess) return cuda_fail(e, "peer store");
    cudaEventRecord(J.ev_b[src], S.s_mig);
    Slot& T = slot_of(rt, target);
    if (T.remote) {
      // process-per-GPU handoff: the copy must be complete before the partner adopts the job
      if ((e = wait_event_relaxed(J.ev_b[src])) != cudaSuccess) return cuda_fail(e, "peer store wait");
      const float us = static_cast<float>(tstamp_us(S.tstamp));
      if (rt->cfg.poison_released) {
        if ((e = poison(B, S.s_mig)) != cudaSuccess) return cuda_fail(e, "poison");
        if ((e = cudaStreamSynchronize(S.s_mig)) != cudaSuccess) return cuda_fail(e, "poison sync");
      }
      lk.lock();
      J.mig_enqueued = true;
      J.dev = target;
      J.n_preempt++;
      J.migrated += g.live_bytes[k];
      J.pack_us = 0.0;
      J.unpack_us = 0.0;
      J.xfer_us = us >= 0.f ? us : elapsed_us(J.ev_a[src], J.ev_b[src]);
      J.state = SF_JOB_MIGRATED_OUT;
      rt->cv.notify_all();
      return SF_OK;
    }
    // stream-ordered resume: the target's training stream waits on the source's copy
    // (a cross-device event wait when the slots are different GPUs)
    e = cudaStreamWaitEvent(T.s_train, J.ev_b[src], 0);
    if (e != cudaSuccess) return cuda_fail(e, "stream wait");
    // as for the host tier: relaunch only once the state has landed on the target
    if ((e = wait_event_relaxed(J.ev_b[src])) != cudaSuccess) return cuda_fail(e, "peer store wait");
    if (rt->cfg.poison_released) {
      if ((e = poison(B, S.s_mig)) != cudaSuccess) return cuda_fail(e, "poison");
    }
    lk.lock();
    J.mig_enqueued = true;
    J.dev = target;
    if (expl) {
      J.state = SF_JOB_PREEMPTED;
      rt->cv.notify_all();
      rt->cv.wait(lk, [&] { return J.resume_req || J.stop_req || rt->shutting_down; });
      if (!J.resume_req) { J.state = SF_JOB_DONE; rt->cv.notify_all(); return SF_OK; }
      J.resume_req = false;
    }
  }
  J.n_preempt++;
  J.migrated += g.live_bytes[k];
  J.state = SF_JOB_RUNNING;
  J.stamp_resume = true;
  rt->cv.notify_all();
  return SF_OK;
}

// ---- host feeds (rt->m held) -----------------------------------------------------------
// A shared-feed member takes part in the lockstep until its job finished; a member whose job
// has not started yet is waited for.
bool member_active(const Feed& F, int m) {
  const Job* j = F.member_jobs[m];
  if (!j) return true;
  if (j->state == SF_JOB_DONE || j->state == SF_JOB_FAILED || j->state == SF_JOB_MIGRATED_OUT) return false;
  return !(j->k == 0 && (j->it >= j->iters || j->stop_req));
}
// Shared slots whose batch every active member has copied become free for the next batch.
void feed_release_drained(Feed& F) {
  if (!F.shared) return;
  const uint32_t all = F.members.size() >= 32 ? ~0u : (1u << F.members.size()) - 1;
  uint32_t inactive = 0;
  for (size_t m = 0; m < F.members.size(); ++m)
    if (!member_active(F, static_cast<int>(m))) inactive |= 1u << m;
  for (int s = 0; s < F.depth; ++s)
    if (F.slot_state[s] == 2 && (F.consumed[s] | inactive) == all) F.slot_state[s] = 0;
}
// Lockstep round-robin: member 0's iteration i, member 1's, ..., then i + 1.
void feed_advance_turn(Feed& F) {
  const int M = static_cast<int>(F.members.size());
  for (int i = 0; i < M; ++i) {
    if (++F.turn_m == M) { F.turn_m = 0; ++F.turn_it; }
    if (member_active(F, F.turn_m)) return;
  }
}
// S_0 of iteration `it` retired: its copy of the slot into the arena has executed.
void feed_consumed(Feed& F, int64_t it, int member) {
  const int s = static_cast<int>(it % F.depth);
  if (F.slot_iter[s] != it || F.slot_state[s] != 2) return;
  if (!F.shared) {
    F.slot_state[s] = 0;
  } else {
    F.consumed[s] |= 1u << member;
    feed_release_drained(F);
  }
}
void push_host_event(sf_runtime* rt, const Feed& F, int job, int64_t it, uint64_t t0, uint64_t t1) {
  sf_trace_event ev{};
  ev.dev = -1 - static_cast<int32_t>(F.id);
  ev.job = job;
  ev.kind = SF_EV_HOST;
  ev.k = -1;
  ev.iter = it;
  ev.t0_ns = t0;
  ev.t1_ns = t1;
  ev.arrival_ns = t0;
  push_trace(rt, ev);
}
// Run the host stage for iteration `it` into ring slot s (rt->m NOT held); "" on success.
std::string feed_fill(sf_runtime* rt, Feed& F, int s, int64_t it) {
  std::vector<void*> dst(F.n);
  for (int i = 0; i < F.n; ++i) dst[i] = F.host + s * F.stride + F.off[i];
  if (F.fn(F.user, it, dst.data(), F.bytes.data(), F.n) != 0) return "host stage returned an error";
  if (F.shared) {  // the immutable device copy every member reads (members' training streams
                   // wait for ev[s]; the slot is refilled only after all of them consumed it)
    cudaError_t e = cudaSetDevice(rt->slots[F.dev]->cuda);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(F.dbuf + s * F.stride, F.host + s * F.stride, F.stride, cudaMemcpyHostToDevice, F.st);
    if (e == cudaSuccess) e = cudaEventRecord(F.ev[s], F.st);
    if (e != cudaSuccess) return std::string("feed H2D: ") + cudaGetErrorString(e);
  }
  return "";
}

// The feed's CPU executor: prefetches up to `depth` iterations, never holding a device.
void stager_main(sf_runtime* rt, Feed* Fp) {
  Feed& F = *Fp;
  std::unique_lock<std::mutex> lk(rt->m);
  while (true) {
    rt->cv.wait(lk, [&] {
      return rt->shutting_down || F.failed ||
             (F.active && !F.inline_mode && F.slot_state[F.next_iter % F.depth] == 0);
    });
    if (rt->shutting_down || F.failed) break;
    const int64_t it = F.next_iter;
    const int s = static_cast<int>(it % F.depth);
    const uint64_t gen = F.gen;
    F.slot_state[s] = 1;
    F.slot_iter[s] = it;
    F.consumed[s] = 0;
    ++F.next_iter;
    lk.unlock();
    const uint64_t t0 = now_ns();
    const std::string err = feed_fill(rt, F, s, it);
    const uint64_t t1 = now_ns();
    lk.lock();
    if (!err.empty()) {
      F.failed = true;
      F.error = err;
      rt->cv.notify_all();
      break;
    }
    F.slot_state[s] = gen == F.gen ? 2 : 0;  // a restart meanwhile discards the fill
    push_host_event(rt, F, static_cast<int>((1u << 21) | F.id), it, t0, t1);
    rt->cv.notify_all();
  }
}

// Job driver.  J.it / J.k is the LAUNCH cursor (the next subgraph not yet launched); up to
// max_inflight subgraphs are queued on the device back to back (no host gap between them).
// When a preemption is requested or a request is queued on the device, launching stops,
// the in-flight subgraphs finish (dispatched kernels are allowed to
// finish), and the cut is taken at the cursor.
void driver_main(sf_runtime* rt, Job* Jp) {
  Job& J = *Jp;
  Graph& g = *J.g;
  const int n = static_cast<int>(g.parts.size());
  const int W = std::max(1, std::min(rt->cfg.max_inflight, kMaxInflight));
  struct Inflight {
    int64_t it;
    int k, dev, ev;
    uint64_t t0;
    bool stamp;
  };
  std::deque<Inflight> q;
  // device-time estimate per subgraph (EMA of host-observed busy intervals); with
  // inflight_budget_us > 0 a subgraph is queued behind others only while the queued work
  // stays within the budget, which bounds the drain a preemption waits for.  The budget is
  // time-aware: the front subgraph counts only its estimated REMAINING time (it started at
  // front_start, when its predecessor was seen to finish, or at its dispatch), so the next one
  // is queued while the front still runs instead of after a host round trip.
  std::vector<double> est_us(n, 0.0);
  const double budget_us = rt->cfg.inflight_budget_us;
  uint64_t front_start = 0;  // host estimate of the front's device start (0: unknown)
  auto queued_us = [&] {
    double t = 0.0;
    for (const auto& f : q) t += est_us[f.k];
    if (!q.empty() && front_start) {
      const double el = (now_ns() - front_start) * 1e-3;
      t -= std::min(est_us[q.front().k], std::max(0.0, el));
    }
    return t;
  };
  int ev_next = 0;
  uint64_t last_t1 = 0;
  // Retired subgraphs whose device interval is mapped later: the timing-event reads (anchor
  // lookups + cudaEventElapsedTime, several us) run while the GPU executes the next subgraph
  // instead of between the completion and the next launch.  Flushed, in retire order, at the
  // start of the next retire wait and when the job ends.
  struct PendTrace {
    int dev, ev;
    uint64_t t0;
    sf_trace_event tev;
    double D0, D1;
  };
  std::vector<PendTrace> pend;
  auto map_pend = [&] {  // rt->m NOT held
    for (auto& p : pend) {
      Slot& PS = slot_of(rt, p.dev);
      p.tev.d0_ns = event_host_ns(PS, J.ev_start[p.dev * kEvRing + p.ev], p.t0);
      p.tev.d1_ns = event_host_ns(PS, J.ev_ring[p.dev * kEvRing + p.ev], p.t0);
      p.D0 = event_dev_D(PS, J.ev_start[p.dev * kEvRing + p.ev], p.t0);
      p.D1 = event_dev_D(PS, J.ev_ring[p.dev * kEvRing + p.ev], p.t0);
    }
  };
  auto push_pend = [&] {  // rt->m held
    for (auto& p : pend) push_trace(rt, p.tev, p.D0, p.D1);
    pend.clear();
  };
  auto flush_pend_locked = [&] {  // off the dispatch path (cut, idle waits): rt->m held
    if (pend.empty()) return;
    map_pend();
    push_pend();
  };
  int64_t broke_for = -1;  // front (it * n + k) whose wait was left early once
  std::unique_lock<std::mutex> lk(rt->m);
  bool pending_peer_stats = false;
  int stats_slot = -1;
  auto release = [&] {
    if (J.holds_token) {
      Slot& S = slot_of(rt, J.dev);
      if (S.owner == static_cast<int>(J.id)) S.owner = -1;
      J.holds_token = false;
      rt->cv.notify_all();
    }
  };
  while (true) {
    if (J.state == SF_JOB_FAILED) break;
    bool launch = false;
    const bool finished = J.it >= J.iters || (J.stop_req && J.k == 0) || rt->shutting_down;
    if (finished) {
      if (q.empty()) {
        if (!pend.empty()) {
          lk.unlock();
          map_pend();
          lk.lock();
          push_pend();
        }
        release();
        J.state = SF_JOB_DONE;
        if (g.feed) {
          Feed& F = *g.feed;
          bool any = false;
          if (F.shared) {  // leave the lockstep
            if (F.turn_m == g.feed_member) feed_advance_turn(F);
            for (size_t m = 0; m < F.members.size(); ++m) any |= member_active(F, static_cast<int>(m));
          }
          if (!any) F.active = false;  // the stage stops prefetching
          else feed_release_drained(F);
        }
        rt->cv.notify_all();
        break;
      }
    } else {
      // boundary gate at the launch cursor
      const bool at_cut_ok = !rt->cfg.iteration_granularity || J.k == 0;
      if (!J.preempt_req && J.sched_pos < J.sched.size() && J.sched[J.sched_pos].iter == J.it &&
          J.sched[J.sched_pos].k == J.k) {
        J.preempt_req = J.sched[J.sched_pos].target != J.dev;  // a move to itself is a no-op
        J.preempt_park = false;
        J.preempt_target = J.sched[J.sched_pos].target;
        J.t_req = now_ns();
        ++J.sched_pos;
      }
      // the device is wanted by queued inference (always first, Q13) or by a present
      // higher-priority training job
      const bool req_inf = slot_has_inference(rt, J.dev);
      const Job* hp = req_inf ? nullptr : higher_training(rt, J, J.dev);
      const bool has_inf = req_inf || hp != nullptr;
      if (J.gate_cut_pending && J.auto_target == J.dev) J.gate_cut_pending = false;  // waits in place
      const bool auto_want = rt->cfg.auto_preempt && rt->cfg.exclusive_gpu &&
                             (has_inf || J.gate_cut_pending) && J.auto_target != J.dev;
      // migrate_home: back to the start slot once it is free (no inference queued there, no
      // present job of priority >= ours); a peer move like any other
      const bool home_want = rt->cfg.migrate_home && !has_inf && J.dev != J.home &&
                             g.bind[J.home] && !g.bind[J.home]->remote &&
                             g.bind[J.dev]->peer.count(J.home) && !slot_has_inference(rt, J.home) &&
                             !present_job(rt, J.home, &J, J.g->priority, true) &&
                             (!rt->cfg.iteration_granularity || J.k == 0);
      const bool want_cut = J.preempt_req || (auto_want && at_cut_ok) || home_want;
      // without a migration, yield the device to queued inference at this boundary (unless the
      // session-slicing baseline keeps it for the rest of the iteration)
      const bool yield_to_inf = rt->cfg.exclusive_gpu && has_inf && !(auto_want && !at_cut_ok);
      if (want_cut) {
        if (q.empty()) {
          release();
          if (!J.preempt_req) {
            J.preempt_park = false;
            J.preempt_target = home_want ? J.home : J.auto_target;
            J.t_req = J.gate_cut_pending ? J.gate_t_req
                      : req_inf ? slot_of(rt, J.dev).q.front()->arrival
                      : hp ? hp->t_submit : now_ns();
          }
          J.gate_cut_pending = false;
          const int src = J.dev;
          const bool peer = J.preempt_target != SF_TARGET_HOST;
          flush_pend_locked();
          if (do_preempt(rt, J, lk) != SF_OK) break;
          if (J.state == SF_JOB_DONE || J.state == SF_JOB_MIGRATED_OUT) break;
          if (peer) { pending_peer_stats = true; stats_slot = src; }
          continue;
        }
      } else if (yield_to_inf) {
        if (q.empty()) {
          release();
          flush_pend_locked();
          rt->cv.wait(lk);
          continue;
        }
      } else {
        Slot& S = slot_of(rt, J.dev);
        // host feed: S_0 needs its iteration's inputs (shared feed: also its lockstep turn);
        // until then the job leaves the device to others — one job's CPU stage overlaps
        // another job's GPU subgraphs
        bool feed_ok = true;
        if (g.feed && J.k == 0) {
          Feed& F = *g.feed;
          if (F.failed) {
            release();
            J.error = "host stage: " + F.error;
            J.state = SF_JOB_FAILED;
            rt->cv.notify_all();
            break;
          }
          const int s = static_cast<int>(J.it % F.depth);
          if (F.shared && !(F.turn_it == J.it && F.turn_m == g.feed_member)) feed_ok = false;
          else if (!F.inline_mode && !(F.slot_state[s] == 2 && F.slot_iter[s] == J.it)) feed_ok = false;
        }
        if (!feed_ok) {
          if (q.empty()) {
            release();
            flush_pend_locked();
            rt->cv.wait(lk);
            continue;
          }
        } else if (rt->cfg.exclusive_gpu && !J.holds_token) {
          // invariant 1: no other model's subgraph on this device
          if (S.owner != -1) {
            if (q.empty()) {
              flush_pend_locked();
              rt->cv.wait(lk);
              continue;
            }
          } else {
            S.owner = static_cast<int>(J.id);
            J.holds_token = true;
          }
        }
        launch = feed_ok && (!rt->cfg.exclusive_gpu || J.holds_token) && static_cast<int>(q.size()) < W &&
                 (q.empty() || budget_us <= 0.0 || queued_us() + est_us[J.k] <= budget_us);
      }
    }
    if (launch) {
      Slot& S = slot_of(rt, J.dev);
      const int dev = J.dev, k = J.k;
      const int64_t it = J.it;
      cudaGraphExec_t ver = g.bind[dev]->versions[k];
      sfk::count_launch(g.bind[dev]->version_kernels[k]);
      Feed* F = k == 0 ? g.feed : nullptr;
      const int fslot = F ? static_cast<int>(it % F->depth) : -1;
      J.launching = true;  // until the launch below is registered (early-launch handshake)
      if (F && F->inline_mode && !(F->slot_state[fslot] == 2 && F->slot_iter[fslot] == it)) {
        // session-slicing baseline: the CPU stage runs now, while the job holds the device
        F->slot_state[fslot] = 1;
        F->slot_iter[fslot] = it;
        lk.unlock();
        const uint64_t h0 = now_ns();
        const std::string err = feed_fill(rt, *F, fslot, it);
        const uint64_t h1 = now_ns();
        lk.lock();
        if (!err.empty()) {
          J.launching = false;
          release();
          J.error = "host stage: " + err;
          J.state = SF_JOB_FAILED;
          rt->cv.notify_all();
          break;
        }
        F->slot_state[fslot] = 2;
        push_host_event(rt, *F, static_cast<int>(J.id), it, h0, h1);
      }
      const bool stamp = J.stamp_resume;
      J.stamp_resume = false;
      // drain gate: a subgraph queued behind an in-flight one waits on the slot's gate word, so
      // a request arriving meanwhile can run before it (reading Q38)
      const bool gated = rt->cfg.drain_gate && S.gate && !q.empty();
      const uint32_t ticket = S.next_ticket++;
      if (rt->cfg.drain_gate && S.gate && !S.gate_held && (ticket & 0xFFFFF) == 0) gate_open(S);
      const int ev = ev_next;
      ev_next = (ev_next + 1) % (2 * W);
      const uint64_t t0 = now_ns();  // decision time, under the lock (trace superset interval)
      lk.unlock();
      cudaSetDevice(S.cuda);
      // resume point: everything stream-ordered before it (H2D + unpack, or the cross-slot
      // wait on the peer store) has executed when this event completes on the device
      cudaError_t e = stamp ? cudaEventRecord(J.ev_r[dev], S.s_train) : cudaSuccess;
      if (e == cudaSuccess && gated) {
        // A = t (posted write), then wait until (int32)(G - t) >= 0: the GPU's read of G cannot
        // pass its write of A on PCIe, which the dispatcher's hold handshake relies on
        if (write_value32()(reinterpret_cast<CUstream>(S.s_train), S.gate_A, ticket, 0) != CUDA_SUCCESS ||
            wait_value32()(reinterpret_cast<CUstream>(S.s_train), S.gate_G, ticket, CU_STREAM_WAIT_VALUE_GEQ) !=
                CUDA_SUCCESS)
          e = cudaErrorLaunchFailure;
      }
      if (e == cudaSuccess) e = cudaEventRecord(J.ev_start[dev * kEvRing + ev], S.s_train);
      if (e == cudaSuccess && F) {  // this iteration's fed tensors into the arena, then S_0
        const uint8_t* src = (F->shared ? F->dbuf : F->host) + fslot * F->stride;
        uint8_t* arena = g.bind[dev]->arena;
        if (F->shared) e = cudaStreamWaitEvent(S.s_train, F->ev[fslot], 0);
        for (int i = 0; e == cudaSuccess && i < F->n; ++i)
          e = cudaMemcpyAsync(arena + g.T[g.feed_tids[i]].offset, src + F->off[i], F->bytes[i],
                              cudaMemcpyDefault, S.s_train);
      }
      if (e == cudaSuccess) e = cudaGraphLaunch(ver, S.s_train);
      if (e == cudaSuccess) e = cudaEventRecord(J.ev_ring[dev * kEvRing + ev], S.s_train);
      lk.lock();
      J.launching = false;
      if (e != cudaSuccess) {
        release();
        J.error = std::string("subgraph launch: ") + cudaGetErrorString(e);
        J.state = SF_JOB_FAILED;
        rt->cv.notify_all();
        break;
      }
      if (q.empty()) front_start = t0;
      q.push_back({it, k, dev, ev, t0, stamp});
      J.infl.push_back({ticket, gated, J.ev_ring[dev * kEvRing + ev]});
      J.last_ev = J.ev_ring[dev * kEvRing + ev];
      J.n_inflight = static_cast<int>(q.size());
      if (S.qn.load(std::memory_order_acquire) > 0) rt->cv.notify_all();  // a waiting dispatcher
      if (++J.k == n) {
        J.k = 0;
        ++J.it;
        if (g.feed && g.feed->shared) {  // the next member's turn on this batch
          feed_advance_turn(*g.feed);
          rt->cv.notify_all();
        }
      }
      continue;
    }
    if (q.empty()) {  // nothing launched and nothing in flight: wait for a state change
      flush_pend_locked();
      rt->cv.wait(lk);
      continue;
    }
    // retire the oldest in-flight subgraph
    const Inflight f = q.front();
    Slot& S = slot_of(rt, f.dev);
    // time-aware budget: leave the wait (once per front) when the next subgraph fits the
    // budget while the front is still running; the gate at the top decides under the lock
    const bool may_break = budget_us > 0.0 && static_cast<int>(q.size()) < W && !J.preempt_req &&
                           J.it < J.iters && !J.stop_req && !(g.feed && J.k == 0) &&
                           broke_for != (f.it * n + f.k);
    lk.unlock();
    cudaSetDevice(S.cuda);
    map_pend();  // the previous retire's device interval, while this front runs
    uint64_t t_res = 0;
    cudaError_t e = cudaSuccess;
    bool broke = false;
    for (;;) {
      if (f.stamp && !t_res && cudaEventQuery(J.ev_r[f.dev]) == cudaSuccess) t_res = now_ns();
      const cudaError_t qq = cudaEventQuery(J.ev_ring[f.dev * kEvRing + f.ev]);
      if (qq == cudaErrorNotReady) {
        const bool req_waiting = S.qn.load(std::memory_order_relaxed) > 0;
        if (may_break && !req_waiting && queued_us() + est_us[J.k] <= budget_us) {
          broke = true;
          break;
        }
        // pause between polls; back off further while a request is queued: its dispatcher is
        // launching the chain and the driver lock is the contended resource (~5 us per poll)
        for (int i = 0, n = req_waiting ? 256 : 16; i < n; ++i) cpu_relax();
        continue;
      }
      e = qq;
      break;
    }
    if (broke) {
      broke_for = f.it * n + f.k;
      lk.lock();
      push_pend();
      continue;
    }
    const uint64_t t1 = now_ns();
    if (f.stamp && !t_res) t_res = t1;
    // device execution interval on the host clock (0 when no anchor covers it)
    uint64_t d0 = 0, d1 = 0;
    double D0 = std::nan(""), D1 = std::nan("");
    if (e == cudaSuccess && f.stamp) {  // others: deferred (pend)
      d0 = event_host_ns(S, J.ev_start[f.dev * kEvRing + f.ev], f.t0);
      d1 = event_host_ns(S, J.ev_ring[f.dev * kEvRing + f.ev], f.t0);
      D0 = event_dev_D(S, J.ev_start[f.dev * kEvRing + f.ev], f.t0);
      D1 = event_dev_D(S, J.ev_ring[f.dev * kEvRing + f.ev], f.t0);
      if (f.stamp) {  // the resume point as the GPU saw it
        const uint64_t r = event_host_ns(S, J.ev_r[f.dev], f.t0);
        if (r) t_res = r;
      }
    }
    float unpack_us = -1.f, h2d_us = 0.f, peer_us = -1.f;
    if (e == cudaSuccess && f.stamp && J.adopted_pending) {
      J.adopted_pending = false;  // the copy was timed by the exporting process
    } else if (e == cudaSuccess && f.stamp) {
      if (pending_peer_stats) {
        peer_us = static_cast<float>(tstamp_us(slot_of(rt, stats_slot).tstamp));
        if (peer_us < 0.f) peer_us = elapsed_us(J.ev_a[stats_slot], J.ev_b[stats_slot]);
        pending_peer_stats = false;
      } else {
        h2d_us = elapsed_us(J.ev_a[f.dev], J.ev_b[f.dev]);
        unpack_us = static_cast<float>(tstamp_us(S.tstamp + 2));
        if (unpack_us < 0.f) unpack_us = elapsed_us(J.ev_b[f.dev], J.ev_c[f.dev]);
      }
    }
    lk.lock();
    push_pend();
    q.pop_front();
    if (!J.infl.empty()) J.infl.pop_front();
    J.n_inflight = static_cast<int>(q.size());
    if (f.k == 0 && g.feed) feed_consumed(*g.feed, f.it, g.feed_member);
    if (f.stamp) {
      J.last_resume = t_res;  // host-observed device resume (CLOCK_MONOTONIC)
      if (unpack_us >= 0.f) { J.unpack_us = unpack_us; J.xfer_us += std::max(h2d_us, 0.f); }
      if (peer_us >= 0.f) { J.pack_us = 0.0; J.xfer_us = peer_us; J.unpack_us = 0.0; }
    }
    if (e != cudaSuccess) {
      release();
      J.error = std::string("subgraph: ") + cudaGetErrorString(e);
      J.state = SF_JOB_FAILED;
      rt->cv.notify_all();
      break;
    }
    sf_trace_event tev{};
    tev.dev = f.dev; tev.job = static_cast<int32_t>(J.id); tev.kind = SF_EV_TRAIN; tev.k = f.k;
    tev.iter = f.it;
    tev.t0_ns = std::max(f.t0, last_t1);  // queued behind its predecessor on the stream
    tev.t1_ns = t1;
    tev.d0_ns = d0;
    tev.d1_ns = d1;
    {
      const double d = (t1 - tev.t0_ns) * 1e-3;
      est_us[f.k] = est_us[f.k] > 0.0 ? 0.75 * est_us[f.k] + 0.25 * d : d;
    }
    tev.arrival_ns = f.t0;  // train events: host dispatch (launch) time
    last_t1 = t1;
    front_start = q.empty() ? 0 : std::max(q.front().t0, t1);
    if (f.stamp) push_trace(rt, tev, D0, D1);
    else pend.push_back({f.dev, f.ev, f.t0, tev, D0, D1});
    // iteration-granularity (session time slicing baseline) keeps the device for the whole
    // iteration; otherwise an empty window is a scheduling point
    if (q.empty() && (!rt->cfg.iteration_granularity || J.k == 0)) release();
    rt->cv.notify_all();
  }
}

// Refreshes every local slot's clock anchor every 200 ms (float elapsed times stay exact to
// well under 1 us; offset drift between the GPU timer and CLOCK_MONOTONIC is re-measured).
void clock_main(sf_runtime* rt) {
  std::unique_lock<std::mutex> lk(rt->m);
  while (!rt->shutting_down) {
    rt->cv.wait_for(lk, std::chrono::milliseconds(50), [&] { return rt->shutting_down; });
    if (rt->shutting_down) break;
    lk.unlock();
    for (auto& S : rt->slots)
      if (!S->remote && refresh_anchor(*S) != cudaSuccess) cudaGetLastError();
    lk.lock();
  }
}

void dispatcher_main(sf_runtime* rt, Slot* S) {
  cudaSetDevice(S->cuda);
  std::unique_lock<std::mutex> lk(rt->m);
  const bool excl = rt->cfg.exclusive_gpu != 0;
  const int64_t spin_us = rt->cfg.dispatch_spin_us;
  auto free_for_inference = [&] {
    const int o = S->owner.load(std::memory_order_acquire);
    return !excl || o == -1 || o == kInferOwner;
  };
  // Early launch (cfg.early_launch): the request need not wait on the host for the training
  // job's in-flight subgraphs to drain.  Once the job's driver can dispatch nothing more (its
  // boundary gate sees the queued request, and it is not inside a launch), the dispatcher
  // takes the device token and enqueues the chain behind a stream-ordered wait on the job's
  // newest in-flight subgraph: the GPU starts the preempter the moment the preemptee's
  // dispatched kernels finish, and the launches overlap that drain ("the preparation of the
  // new job overlaps the abort of the preempted one").  No subgraph of the
  // two models co-runs on the device (invariant 1 holds through the device dependency; the
  // trace records it, oracle/schedule.py I1).  Not with iteration-granularity slicing.
  const bool early = excl && rt->cfg.early_launch && !rt->cfg.iteration_granularity;
  auto steal_from = [&]() -> Job* {  // rt->m held
    if (!early) return nullptr;
    const int o = S->owner.load(std::memory_order_acquire);
    if (o < 0 || o >= kInferOwner || static_cast<size_t>(o) >= rt->jobs.size()) return nullptr;
    Job* J = rt->jobs[o].get();
    return J && !J->launching && J->dev == S->id ? J : nullptr;
  };
  auto ready = [&] {
    return rt->shutting_down || (!S->q.empty() && (free_for_inference() || steal_from() != nullptr));
  };
  while (true) {
    if (!ready() && spin_us != 0) {
      // busy-poll (no futex wake-up on the request path) for dispatch_spin_us, -1 = forever
      const uint64_t deadline = spin_us < 0 ? ~0ull : now_ns() + static_cast<uint64_t>(spin_us) * 1000;
      lk.unlock();
      while (!rt->stop_spin.load(std::memory_order_relaxed) && now_ns() < deadline) {
        if (S->qn.load(std::memory_order_acquire) > 0 && (early || free_for_inference())) break;
        for (int i = 0; i < 32; ++i) cpu_relax();
      }
      lk.lock();
    }
    rt->cv.wait(lk, ready);
    if (S->q.empty() && rt->shutting_down) break;
    if (S->q.empty()) continue;
    Request* r = S->q.front();
    Job* dep = free_for_inference() ? nullptr : steal_from();
    cudaEvent_t dep_ev = nullptr;
    bool held_now = false;
    // a device that looks free may still run a job's subgraphs that a drain-gate hold released
    // when the previous chain ended (the job gave the token up with them in flight): the chain
    // is device-ordered after them as well (invariant 1).  While the gate still holds them
    // (requests queued back to back) they cannot start before it opens after this queue drains,
    // and the running one was waited for by the request that took the hold: no wait (waiting
    // on a held subgraph would deadlock the queue)
    Job* drain = nullptr;
    if (!dep && excl && !S->gate_held) {
      for (auto& jp : rt->jobs) {
        Job* Jx = jp.get();
        if (Jx && Jx->dev == S->id && Jx->n_inflight > 0 && Jx->last_ev) {
          drain = Jx;
          dep_ev = Jx->last_ev;
          break;
        }
      }
    }
    if (dep) {
      dep_ev = dep->n_inflight > 0 ? dep->last_ev : nullptr;
      // drain gate: hold the queued subgraphs (tickets >= the second in flight) so the chain
      // runs right after the RUNNING one.  Dekker handshake: store G = t - 1, full fence, load
      // A.  A still < t: the GPU's read of G (which cannot pass its write of A) comes after our
      // store, so it sees the hold.  Otherwise it may have passed: release, wait for all.
      if (S->gate && dep->infl.size() >= 2 && dep->infl[1].gated && !S->gate_held) {
        const uint32_t t = dep->infl[1].ticket;
        S->gate[0] = t - 1u;
        std::atomic_thread_fence(std::memory_order_seq_cst);
        const uint32_t a = S->gate[16];
        if (static_cast<int32_t>(a - t) < 0) {
          S->gate_held = true;
          held_now = true;
          dep_ev = dep->infl[0].end;
          if (!dep->gate_cut_pending) {
            dep->gate_cut_pending = true;
            dep->gate_t_req = r->arrival;
          }
        } else {
          gate_open(*S);
        }
      }
      dep->holds_token = false;  // the job re-acquires the token before its next launch
      if (r->preempted_job < 0) {
        r->preempted_job = static_cast<int>(dep->id);
        r->cut_iter = dep->it;  // the launch cursor: where the job stops
        r->cut_k = dep->k;
      }
    }
    if (rt->cfg.exclusive_gpu) S->owner = kInferOwner;
    Graph& g = *r->g;
    Binding* B = g.bind[S->id].get();
    const uint64_t t0 = now_ns();
    lk.unlock();
    cudaError_t e = cudaSuccess;
    const Tensor& tin = g.T[g.input_tid];
    const Tensor& tout = g.T[g.output_tid];
    // Request I/O with the SM copy kernel on the high-priority stream: device or pinned
    // (UVA-mapped) host buffers alike, never queued behind a copy-engine migration.
    const bool aligned = reinterpret_cast<uintptr_t>(r->in) % 16 == 0 &&
                         reinterpret_cast<uintptr_t>(r->out) % 16 == 0 && tin.nbytes % 4 == 0 &&
                         tout.nbytes % 4 == 0;
    // Direct launches with programmatic dependent launch (default): each kernel of the chain
    // is scheduled while its predecessor drains and GEMVs stream their (constant) weights
    // before the previous layer finishes; SF_INFER_DIRECT=0 replays the captured versions.
    static const bool direct = !(std::getenv("SF_INFER_DIRECT") && std::getenv("SF_INFER_DIRECT")[0] == '0');
    static const bool use_pdl = !(std::getenv("SF_PDL") && std::getenv("SF_PDL")[0] == '0');
    std::string op_err;
    if (direct) sfk::set_pdl(use_pdl);
    if (direct && S->l2_setaside > 0 && !B->l2_planned) {
      // persisting L2 set-aside: keep whole weight tensors, largest first, within the set-aside
      // (a cyclic stream larger than the set-aside would thrash it); the rest is streamed
      // evict-first so it cannot displace them (reading Q29)
      std::vector<std::pair<uint64_t, int>> ws;
      for (const auto& o : g.ops)
        if (o.type == SF_OP_GEMM && !g.op_written[o.in[1]] && g.T[o.out[0]].rows <= 8)
          ws.push_back({g.T[o.in[1]].nbytes, o.in[1]});
      std::sort(ws.rbegin(), ws.rend());
      uint64_t used = 0;
      for (auto [nb, t] : ws)
        if (used + nb <= S->l2_setaside) { B->l2_keep.insert(t); used += nb; }
      B->l2_planned = true;
    }
    // device-resident request buffers are read / written in place by the kernels (saving the
    // two copy kernels of the I/O staging); pinned host buffers keep the SM copy kernels, which
    // move them in one coalesced pass instead of every GEMV CTA reading its x slice over PCIe
    static const bool redirect = !(std::getenv("SF_INFER_REDIRECT") && std::getenv("SF_INFER_REDIRECT")[0] == '0');
    auto on_device = [](const void* p) {
      cudaPointerAttributes a{};
      if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
      }
      return a.type == cudaMemoryTypeDevice;
    };
    if (direct && infer_graph_mode() && B->rg.state == 0 && B->blocked_ready) build_req_graph(g, *B, use_pdl);
    const bool use_graph = direct && infer_graph_mode() && B->rg.state == 1 && aligned &&
                           (infer_graph_mode() == 1 || dep_ev == nullptr);
    const bool in_place = direct && aligned && redirect && !use_graph && on_device(r->in) && on_device(r->out);
    // blocked copies of the constant GEMV weights (allocated at bind; laid out here at the first
    // request unless sf_refresh_constants already did it; reading Q39)
    if (!B->blocked_ready) {
      layout_blocked(g, *B, S->s_infer);
      B->blocked_ready = true;
    }
    const uint64_t tl0 = now_ns();
    // early launch: the chain (and its start event) wait on the device for the job's
    // dispatched subgraphs; the driver dispatches nothing more while the request is queued
    if (dep_ev) e = cudaStreamWaitEvent(S->s_infer, dep_ev, 0);
    if (e == cudaSuccess) e = cudaEventRecord(S->ev_i0, S->s_infer);
    if (e != cudaSuccess || in_place || use_graph) {
    } else if (aligned) {
      e = sfk::launch_copy(r->in, B->arena + tin.offset, tin.nbytes, S->s_infer);
    } else {
      e = cudaMemcpyAsync(B->arena + tin.offset, r->in, tin.nbytes, cudaMemcpyDefault, S->s_infer);
    }
    if (use_graph && e == cudaSuccess) e = launch_req_graph(*B, tin, tout, r->in, r->out, S->s_infer);
    for (size_t k = 0; !use_graph && e == cudaSuccess && k < B->versions.size(); ++k) {
      if (direct) {
        Capture c{g, *B, S->s_infer, false, &B->prepared};
        if (S->l2_setaside > 0) c.l2_keep = &B->l2_keep;
        if (in_place) {
          c.redir_in = g.input_tid;
          c.in_ptr = static_cast<uint8_t*>(const_cast<void*>(r->in));
          c.redir_out = g.output_tid;
          c.out_ptr = static_cast<uint8_t*>(r->out);
        }
        if (launch_subgraph_ops(c, static_cast<int>(k)) != SF_OK) {
          op_err = g_err;
          e = cudaErrorUnknown;
        }
      } else {
        e = cudaGraphLaunch(B->versions[k], S->s_infer);
        sfk::count_launch(B->version_kernels[k]);
      }
    }
    if (e == cudaSuccess && !in_place && !use_graph) {
      if (aligned) e = sfk::launch_copy(B->arena + tout.offset, r->out, tout.nbytes, S->s_infer);
      else e = cudaMemcpyAsync(r->out, B->arena + tout.offset, tout.nbytes, cudaMemcpyDefault, S->s_infer);
    }
    const uint64_t tl1 = now_ns();
    sfk::set_pdl(false);
    if (e == cudaSuccess) e = cudaEventRecord(S->ev_infer, S->s_infer);
    if (e == cudaSuccess && S->gate) {
      // safety valve: streams beyond the device's hardware work queues share a queue, and a
      // held gate wait on the training stream would then also hold a chain queued behind it
      // on the same connection.  A chain not done 5 ms after its launch (~50 us normally)
      // releases the hold; the held subgraph then runs first on that shared queue.
      const uint64_t valve = now_ns() + 5000000;
      for (;;) {
        e = cudaEventQuery(S->ev_infer);
        if (e != cudaErrorNotReady) break;
        if (now_ns() > valve) {
          std::lock_guard<std::mutex> vk(rt->m);
          if (S->gate_held) {
            gate_open(*S);
            ++S->gate_valve;
          }
          e = spin_event(S->ev_infer);
          break;
        }
      }
    } else if (e == cudaSuccess) {
      e = spin_event(S->ev_infer);
    }
    const uint64_t t1 = now_ns();
    float dev_ms = -1.f;
    if (e == cudaSuccess && cudaEventElapsedTime(&dev_ms, S->ev_i0, S->ev_infer) != cudaSuccess) {
      dev_ms = -1.f;
      cudaGetLastError();
    }
    uint64_t d0 = 0, d1 = 0;
    double iD0 = std::nan(""), iD1 = std::nan("");
    if (e == cudaSuccess) {
      d0 = event_host_ns(*S, S->ev_i0, tl0);
      d1 = event_host_ns(*S, S->ev_infer, tl0);
      iD0 = event_dev_D(*S, S->ev_i0, tl0);
      iD1 = event_dev_D(*S, S->ev_infer, tl0);
    }
    lk.lock();
    // start = the request chain's start on the GPU (device clock); without an anchor: an
    // early-launched chain starts when the job's drain completes, taken as completion - device
    // time (never earlier than the true device start)
    r->start = d0 ? d0 : dep && dev_ms >= 0.f ? std::max(t0, t1 - static_cast<uint64_t>(dev_ms * 1e6f)) : t0;
    r->end = t1;
    r->device_us = dev_ms >= 0.f ? dev_ms * 1e3f : -1.f;
    r->launch_us = static_cast<float>((tl1 - tl0) * 1e-3);
    r->dispatch_us = static_cast<float>((tl0 - t0) * 1e-3);
    if (e != cudaSuccess) r->error = op_err.empty() ? cudaGetErrorString(e) : op_err;
    r->done = true;
    S->q.pop_front();
    S->qn.fetch_sub(1);
    sf_trace_event ev{};
    ev.dev = S->id; ev.job = static_cast<int32_t>(kInferOwner | (r->id & 0xFFFFF)); ev.kind = SF_EV_INFER;
    ev.t0_ns = t0; ev.t1_ns = t1; ev.arrival_ns = r->arrival;
    ev.d0_ns = d0; ev.d1_ns = d1;
    ev.iter = dep ? static_cast<int64_t>(dep->id) : drain ? static_cast<int64_t>(drain->id) : -1;  // device-ordered after that job's dispatched subgraphs
    ev.k = held_now ? 1 : 0;  // drain gate: the job's queued subgraphs were held behind this request
    push_trace(rt, ev, iD0, iD1);
    if (rt->cfg.exclusive_gpu && S->q.empty()) S->owner = -1;
    if (S->gate_held && S->q.empty()) gate_open(*S);  // the held subgraphs run now
    rt->cv.notify_all();
  }
}

Graph* get_graph(sf_runtime* rt, sf_graph_id g) {
  return g < rt->graphs.size() ? rt->graphs[g].get() : nullptr;
}
Job* get_job(sf_runtime* rt, sf_job_id j) { return j < rt->jobs.size() ? rt->jobs[j].get() : nullptr; }

}  // namespace

// =========================================================================================
// C ABI
// =========================================================================================
extern "C" {

const char* sf_last_error(void) { return g_err.c_str(); }
int32_t sf_abi_version(void) { return SF_ABI_VERSION; }
uint64_t sf_now_ns(void) { return now_ns(); }
uint64_t sf_kernel_launches(void) { return sfk::launches(); }

sf_status sf_create(const sf_config* cfg, sf_runtime** out) {
  if (!cfg || !out || cfg->n_devices <= 0 || !cfg->cuda_ordinals) return fail(SF_EINVAL, "bad config");
  int ndev = 0;
  SF_CK(cudaGetDeviceCount(&ndev));
  auto rt = std::make_unique<sf_runtime>();
  rt->cfg = *cfg;
  rt->cfg.cuda_ordinals = nullptr;
  if (cfg->trace_capacity > 0) rt->trace_cap = static_cast<size_t>(cfg->trace_capacity);
  rt->trace.reserve(std::min<size_t>(rt->trace_cap, 1 << 16));
  for (int s = 0; s < cfg->n_devices; ++s) {
    const int c = cfg->cuda_ordinals[s];
    if (c == -1) {
      auto S = std::make_unique<Slot>();
      S->id = s;
      S->cuda = -1;
      S->remote = true;
      rt->slots.push_back(std::move(S));
      continue;
    }
    if (c < 0 || c >= ndev) return fail(SF_EINVAL, "cuda ordinal out of range");
    auto S = std::make_unique<Slot>();
    S->id = s;
    S->cuda = c;
    SF_CK(cudaSetDevice(c));
    int lo = 0, hi = 0;
    SF_CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    SF_CK(cudaStreamCreateWithFlags(&S->s_train, cudaStreamNonBlocking));
    SF_CK(cudaStreamCreateWithPriority(&S->s_infer, cudaStreamNonBlocking, hi));
    SF_CK(cudaStreamCreateWithFlags(&S->s_mig, cudaStreamNonBlocking));
    SF_CK(cudaEventCreate(&S->ev_infer));
    SF_CK(cudaEventCreate(&S->ev_i0));
    SF_CK(cudaMalloc(&S->tstamp, 4 * sizeof(unsigned long long)));
    SF_CK(cudaStreamCreateWithPriority(&S->s_clk, cudaStreamNonBlocking, hi));
    SF_CK(cudaHostAlloc(reinterpret_cast<void**>(&S->clk_host), 64, cudaHostAllocMapped | cudaHostAllocPortable));
    SF_CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&S->clk_dev), S->clk_host, 0));
    SF_CK(refresh_anchor(*S));
    if (cfg->drain_gate) {
      if (!wait_value32() || !write_value32()) return fail(SF_EUNSUPPORTED, "stream memory operations unavailable");
      void* gp = nullptr;
      SF_CK(cudaHostAlloc(&gp, 128, cudaHostAllocMapped | cudaHostAllocPortable));
      std::memset(gp, 0, 128);
      S->gate = static_cast<volatile uint32_t*>(gp);
      void* dp = nullptr;
      SF_CK(cudaHostGetDevicePointer(&dp, gp, 0));
      S->gate_G = reinterpret_cast<CUdeviceptr>(dp);
      S->gate_A = reinterpret_cast<CUdeviceptr>(dp) + 64;
      gate_open(*S);
    }
    if (cfg->infer_l2_persist_bytes > 0) {
      int mx = 0, mw = 0;
      SF_CK(cudaDeviceGetAttribute(&mx, cudaDevAttrMaxPersistingL2CacheSize, c));
      SF_CK(cudaDeviceGetAttribute(&mw, cudaDevAttrMaxAccessPolicyWindowSize, c));
      S->l2_setaside = std::min<size_t>(cfg->infer_l2_persist_bytes, static_cast<size_t>(mx));
      S->l2_max_window = static_cast<size_t>(mw);
      SF_CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, S->l2_setaside));
    }
    rt->slots.push_back(std::move(S));
  }
  // peer access between distinct physical devices (NVLink / NVSwitch)
  for (auto& a : rt->slots)
    for (auto& b : rt->slots)
      if (!a->remote && !b->remote && a->cuda != b->cuda) {
        int can = 0;
        SF_CK(cudaDeviceCanAccessPeer(&can, a->cuda, b->cuda));
        if (!can) return fail(SF_EUNSUPPORTED, "no peer access between devices");
        SF_CK(cudaSetDevice(a->cuda));
        cudaError_t e = cudaDeviceEnablePeerAccess(b->cuda, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
          return fail(SF_ECUDA, std::string("enable peer access: ") + cudaGetErrorString(e));
        cudaGetLastError();
      }
  sf_runtime* p = rt.release();
  for (auto& S : p->slots)
    if (!S->remote) S->dispatcher = std::thread(dispatcher_main, p, S.get());
  p->clk = std::thread(clock_main, p);
  *out = p;
  return SF_OK;
}

void sf_destroy(sf_runtime* rt) {
  if (!rt) return;
  {
    std::unique_lock<std::mutex> lk(rt->m);
    rt->cv.wait(lk, [&] {
      for (auto& S : rt->slots)
        if (!S->q.empty()) return false;
      for (auto& J : rt->jobs)
        if (J->state == SF_JOB_RUNNING || J->state == SF_JOB_STOPPING || J->state == SF_JOB_MIGRATING)
          return false;
      return true;
    });
    rt->shutting_down = true;
    rt->stop_spin = true;
    rt->cv.notify_all();
  }
  for (auto& J : rt->jobs)
    if (J->driver.joinable()) J->driver.join();
  for (auto& S : rt->slots)
    if (S->dispatcher.joinable()) S->dispatcher.join();
  if (rt->clk.joinable()) rt->clk.join();
  for (auto& F : rt->feeds)
    if (F->stager.joinable()) F->stager.join();
  for (auto& F : rt->feeds) {
    if (F->shared) {
      cudaSetDevice(rt->slots[F->dev]->cuda);
      cudaStreamSynchronize(F->st);
      cudaFree(F->dbuf);
      cudaStreamDestroy(F->st);
      for (auto e : F->ev) cudaEventDestroy(e);
    }
    cudaFreeHost(F->host);
  }
  for (auto& S : rt->slots) {
    if (S->remote) continue;
    cudaSetDevice(S->cuda);
    cudaDeviceSynchronize();
  }
  for (auto& G : rt->graphs)
    for (auto& B : G->bind) {
      if (!B) continue;
      if (B->remote) {
        if (B->ipc_base) {
          cudaSetDevice(B->ipc_device);
          cudaIpcCloseMemHandle(B->ipc_base);
        }
        continue;
      }
      cudaSetDevice(rt->slots[B->slot]->cuda);
      for (auto v : B->versions) cudaGraphExecDestroy(v);
      if (B->rg.exec) cudaGraphExecDestroy(B->rg.exec);
      if (B->rg.graph) cudaGraphDestroy(B->rg.graph);
      for (void* d : B->dev_allocs) cudaFree(d);
      if (B->ws) cudaFree(B->ws);
      if (B->counters) cudaFree(B->counters);
    }
  for (auto& J : rt->jobs)
    for (size_t s = 0; s < J->ev_sub.size(); ++s) {
      if (rt->slots[s]->remote) continue;
      cudaSetDevice(rt->slots[s]->cuda);
      cudaEventDestroy(J->ev_sub[s]);
      cudaEventDestroy(J->ev_r[s]);
      for (int i = 0; i < kEvRing; ++i) {
        cudaEventDestroy(J->ev_ring[s * kEvRing + i]);
        cudaEventDestroy(J->ev_start[s * kEvRing + i]);
      }
      for (int i = 0; i < kCkEvents; ++i) cudaEventDestroy(J->ev_ck[s * kCkEvents + i]);
      cudaEventDestroy(J->ev_a[s]);
      cudaEventDestroy(J->ev_b[s]);
      cudaEventDestroy(J->ev_c[s]);
    }
  for (auto& S : rt->slots) {
    if (S->remote) continue;
    cudaSetDevice(S->cuda);
    cudaStreamDestroy(S->s_train);
    cudaStreamDestroy(S->s_infer);
    cudaStreamDestroy(S->s_mig);
    cudaEventDestroy(S->ev_infer);
    cudaEventDestroy(S->ev_i0);
    cudaFree(S->tstamp);
    for (auto& a : S->anchors) cudaEventDestroy(a.ev);
    cudaStreamDestroy(S->s_clk);
    cudaFreeHost(S->clk_host);
    if (S->gate) cudaFreeHost(const_cast<uint32_t*>(S->gate));
  }
  delete rt;
}

sf_status sf_register_graph(sf_runtime* rt, const sf_graph_desc* gd, int32_t priority,
                            sf_graph_id* out) {
  if (!rt || !gd || !out || (gd->n_tensors && !gd->tensors) || (gd->n_ops && !gd->ops))
    return fail(SF_EINVAL, "null argument");
  auto g = std::make_unique<Graph>();
  g->name = gd->name ? gd->name : "";
  g->priority = priority;
  for (uint32_t i = 0; i < gd->n_tensors; ++i) {
    const sf_tensor_desc& t = gd->tensors[i];
    if (t.rows <= 0 || t.cols <= 0) return fail(SF_EINVAL, "tensor " + std::to_string(i) + ": shape");
    if (t.dtype != SF_F32 && t.dtype != SF_I32) return fail(SF_EUNSUPPORTED, "tensor dtype");
    if (t.kind < SF_PARAM || t.kind > SF_OUTPUT) return fail(SF_EINVAL, "tensor kind");
    g->T.push_back({t.rows, t.cols, t.dtype, t.kind, static_cast<uint64_t>(t.rows) * t.cols * 4, 0});
  }
  g->ops.assign(gd->ops, gd->ops + gd->n_ops);
  if (g->ops.empty()) return fail(SF_EINVAL, "graph has no ops");
  if (sf_status s = validate(*g)) return s;
  for (size_t i = 0; i < g->T.size(); ++i) {
    if (g->T[i].kind == SF_INPUT && g->input_tid < 0) g->input_tid = static_cast<int>(i);
    if (g->T[i].kind == SF_OUTPUT && g->output_tid < 0) g->output_tid = static_cast<int>(i);
  }
  g->op_written.assign(g->T.size(), 0);
  for (const auto& op : g->ops)
    for (int q = 0; q < op.n_out; ++q) g->op_written[op.out[q]] = 1;
  std::lock_guard<std::mutex> lk(rt->m);
  g->bind.resize(rt->slots.size());
  rt->graphs.push_back(std::move(g));
  *out = static_cast<sf_graph_id>(rt->graphs.size() - 1);
  return SF_OK;
}

sf_status sf_partition(sf_runtime* rt, sf_graph_id gid, const sf_partition_opts* o,
                       sf_partition_info* out) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g) return fail(SF_EINVAL, "bad graph id");
  if (g->partitioned) return fail(SF_ESTATE, "graph already partitioned");
  sf_partition_opts def{SF_PART_PER_LAYER_PHASE, 0, 1};
  if (sf_status s = do_partition(*g, o ? *o : def)) return s;
  if (out) {
    out->n_subgraphs = static_cast<int32_t>(g->parts.size());
    out->arena_bytes = g->arena_bytes;
    out->staging_bytes = g->staging_bytes;
    out->persistent_bytes = g->persistent_bytes;
    out->max_live_bytes = g->max_live;
  }
  return SF_OK;
}

sf_status sf_subgraph_range(sf_runtime* rt, sf_graph_id gid, int32_t k, int32_t* b, int32_t* e) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g || !g->partitioned || k < 0 || k >= static_cast<int>(g->parts.size()))
    return fail(SF_EINVAL, "bad graph / cut");
  if (b) *b = g->parts[k].first;
  if (e) *e = g->parts[k].second;
  return SF_OK;
}

sf_status sf_live_set(sf_runtime* rt, sf_graph_id gid, int32_t k, uint32_t* ids, uint32_t cap,
                      uint32_t* n, uint64_t* bytes) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g || !g->partitioned || k < 0 || k >= static_cast<int>(g->parts.size()))
    return fail(SF_EINVAL, "bad graph / cut");
  const auto& L = g->live[k];
  if (n) *n = static_cast<uint32_t>(L.size());
  if (bytes) *bytes = g->live_bytes[k];
  if (ids) std::copy(L.begin(), L.begin() + std::min<size_t>(cap, L.size()), ids);
  return SF_OK;
}

sf_status sf_tensor_offset(sf_runtime* rt, sf_graph_id gid, uint32_t t, uint64_t* off) {
  if (!rt || !off) return fail(SF_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g || !g->partitioned || t >= g->T.size()) return fail(SF_EINVAL, "bad graph / tensor");
  *off = g->T[t].offset;
  return SF_OK;
}

sf_status sf_staging_layout(sf_runtime* rt, sf_graph_id gid, int32_t k, uint64_t* total,
                            uint64_t* offs, uint32_t cap) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g || !g->partitioned || k < 0 || k >= static_cast<int>(g->parts.size()))
    return fail(SF_EINVAL, "bad graph / cut");
  if (total) *total = g->staging_total[k];
  if (offs)
    std::copy(g->payload_off[k].begin(),
              g->payload_off[k].begin() + std::min<size_t>(cap, g->payload_off[k].size()), offs);
  return SF_OK;
}

sf_status sf_bind(sf_runtime* rt, sf_graph_id gid, int32_t dev, void* arena, void* staging,
                  void* host_staging) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* gp = get_graph(rt, gid);
  if (!gp || !gp->partitioned) return fail(SF_ESTATE, "graph not partitioned");
  Graph& g = *gp;
  if (dev < 0 || dev >= static_cast<int>(rt->slots.size())) return fail(SF_EINVAL, "bad slot");
  if (g.bind[dev]) return fail(SF_ESTATE, "slot already bound");
  if (rt->slots[dev]->remote) return fail(SF_EINVAL, "remote slots are mapped with sf_import_arena");
  if (!arena || reinterpret_cast<uintptr_t>(arena) % kAlign)
    return fail(SF_EINVAL, "arena must be a 256-B aligned device pointer");
  if (staging && reinterpret_cast<uintptr_t>(staging) % kAlign)
    return fail(SF_EINVAL, "staging must be 256-B aligned");
  Slot& S = *rt->slots[dev];
  if (rt->cfg.device_budget_bytes &&
      S.persistent_bound + g.persistent_bytes > rt->cfg.device_budget_bytes)
    return fail(SF_ENOMEM, "persistent state of the graphs sharing this device exceeds its budget");
  SF_CK(cudaSetDevice(S.cuda));
  auto b = std::make_unique<Binding>();
  b->slot = dev;
  b->arena = static_cast<uint8_t*>(arena);
  b->staging = static_cast<uint8_t*>(staging);
  b->host_staging = static_cast<uint8_t*>(host_staging);
  if (host_staging) {
    void* dp = nullptr;
    SF_CK(cudaHostGetDevicePointer(&dp, host_staging, 0));
    b->host_staging_dev = static_cast<uint8_t*>(dp);
  }
  for (const auto& op : g.ops) {
    if (op.type != SF_OP_GEMM) continue;
    for (int t : {op.in[0], op.in[1]}) {
      const Tensor& x = g.T[t];
      if (x.kind != SF_DATASET || x.cols % 4 == 0 || b->shadow.count(t)) continue;
      const int pitch = (x.cols + 3) / 4 * 4;
      float* d = nullptr;
      SF_CK(cudaMalloc(&d, static_cast<size_t>(x.rows) * pitch * sizeof(float)));
      SF_CK(cudaMemset(d, 0, static_cast<size_t>(x.rows) * pitch * sizeof(float)));
      b->shadow[t] = {d, pitch};
      b->dev_allocs.push_back(d);
    }
  }
  for (size_t j = 0; j < g.ops.size(); ++j) {
    const sf_op_desc& op = g.ops[j];
    if (op.type != SF_OP_GEMM) continue;
    const Tensor &A = g.T[op.in[0]], &B = g.T[op.in[1]], &C = g.T[op.out[0]];
    const bool ta = op.flags & SF_GEMM_TA, tb = op.flags & SF_GEMM_TB;
    if (C.rows <= 8 && !ta && !tb) continue;  // GEMV path has no pitch requirement
    std::array<Binding::PadBuf, 3> pads{};
    bool any = false;
    const Tensor* ops3[3] = {&A, &B, &C};
    const int ids[3] = {op.in[0], op.in[1], op.out[0]};
    for (int q = 0; q < 3; ++q) {
      const Tensor& x = *ops3[q];
      if (x.cols % 4 == 0 || (q < 2 && b->shadow.count(ids[q]))) continue;
      const int pitch = (x.cols + 3) / 4 * 4;
      float* d = nullptr;
      SF_CK(cudaMalloc(&d, static_cast<size_t>(x.rows) * pitch * sizeof(float)));
      SF_CK(cudaMemset(d, 0, static_cast<size_t>(x.rows) * pitch * sizeof(float)));
      b->dev_allocs.push_back(d);
      pads[q] = {d, pitch};
      any = true;
    }
    if (any) b->gemm_pad[static_cast<int>(j)] = pads;
  }
  if (sf_status s = alloc_blocked(g, *b)) return s;
  SF_CK(cudaMalloc(&b->ws, std::max<uint64_t>(g.ws_floats, 4) * sizeof(float)));
  SF_CK(cudaMalloc(&b->counters, std::max<uint64_t>(g.counter_slots, 1) * sizeof(unsigned)));
  SF_CK(cudaMemset(b->counters, 0, std::max<uint64_t>(g.counter_slots, 1) * sizeof(unsigned)));
  // versions: one CUDA graph per subgraph
  cudaStream_t cap;
  SF_CK(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
  std::map<int, void*>& prepared = b->prepared;
  {
    Capture prep{g, *b, cap, true, &prepared};
    for (size_t k = 0; k < g.parts.size(); ++k)
      if (sf_status s = launch_subgraph_ops(prep, static_cast<int>(k))) { cudaStreamDestroy(cap); return s; }
  }
  for (size_t k = 0; k < g.parts.size(); ++k) {
    SF_CK(cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal));
    Capture c{g, *b, cap, false, &prepared};
    const uint64_t l0 = sfk::launches();
    sf_status s = launch_subgraph_ops(c, static_cast<int>(k));
    const uint64_t nk = sfk::launches() - l0;
    sfk::count_launch(uint64_t(0) - nk);  // captured, not launched: counted at each replay
    cudaGraph_t graph = nullptr;
    cudaError_t e = cudaStreamEndCapture(cap, &graph);
    if (s != SF_OK) { if (graph) cudaGraphDestroy(graph); cudaStreamDestroy(cap); return s; }
    if (e != cudaSuccess) { cudaStreamDestroy(cap); return fail(SF_ECUDA, std::string("capture: ") + cudaGetErrorString(e)); }
    cudaGraphExec_t exec = nullptr;
    e = cudaGraphInstantiate(&exec, graph, 0);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) { cudaStreamDestroy(cap); return fail(SF_ECUDA, std::string("instantiate: ") + cudaGetErrorString(e)); }
    b->versions.push_back(exec);
    b->version_kernels.push_back(nk);
  }
  cudaStreamDestroy(cap);
  // copy lists per cut
  const size_t n = g.parts.size();
  b->pack.resize(n); b->unpack.resize(n); b->pack_zc.resize(n); b->unpack_zc.resize(n);
  for (size_t k = 0; k < n; ++k) {
    void* hdr_dev;
    if (sf_status s = upload(*b, g.header[k].data(), g.header[k].size(), &hdr_dev)) return s;
    for (int mode = 0; mode < 2; ++mode) {
      uint8_t* stg = mode == 0 ? b->staging : b->host_staging_dev;
      if (!stg) continue;
      std::vector<sf_copy_desc> pk, up;
      pk.push_back({hdr_dev, stg, g.payload_start[k], g.payload_start[k]});
      for (size_t e = 0; e < g.live[k].size(); ++e) {
        const Tensor& t = g.T[g.live[k][e]];
        pk.push_back({b->arena + t.offset, stg + g.payload_off[k][e], t.nbytes, round_up(t.nbytes, kAlign)});
        up.push_back({stg + g.payload_off[k][e], b->arena + t.offset, t.nbytes, round_up(t.nbytes, 16)});
      }
      if (sf_status s = build_copy_list(*b, pk, mode == 0 ? &b->pack[k] : &b->pack_zc[k])) return s;
      if (sf_status s = build_copy_list(*b, up, mode == 0 ? &b->unpack[k] : &b->unpack_zc[k])) return s;
    }
  }
  // poison ranges: maximal runs of non-DATASET tensors
  for (size_t t = 0; t < g.T.size();) {
    if (g.T[t].kind == SF_DATASET) { ++t; continue; }
    const uint64_t a = g.T[t].offset;
    size_t u = t;
    while (u < g.T.size() && g.T[u].kind != SF_DATASET) ++u;
    const uint64_t end = (u < g.T.size()) ? g.T[u].offset : g.arena_bytes;
    b->poison_ranges.emplace_back(a, end - a);
    t = u;
  }
  S.persistent_bound += g.persistent_bytes;
  g.bind[dev] = std::move(b);
  // peer lists with every other bound slot, both directions
  for (size_t o = 0; o < g.bind.size(); ++o) {
    if (static_cast<int>(o) == dev || !g.bind[o]) continue;
    if (sf_status s = build_peer_lists(rt, g, *g.bind[dev], *g.bind[o])) return s;
    if (g.bind[o]->remote) continue;  // a remote arena is only ever a destination here
    if (sf_status s = build_peer_lists(rt, g, *g.bind[o], *g.bind[dev])) return s;
  }
  SF_CK(cudaSetDevice(S.cuda));
  SF_CK(cudaDeviceSynchronize());
  return SF_OK;
}

static sf_status start_job(sf_runtime* rt, sf_graph_id gid, int32_t dev, int64_t iters,
                           int32_t auto_target, const sf_cut_request* sched, int32_t n_sched,
                           int64_t it0, int32_t k0, sf_job_id* out) {
  if (!rt || !out || n_sched < 0 || (n_sched > 0 && !sched)) return fail(SF_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g || !g->partitioned) return fail(SF_ESTATE, "graph not partitioned");
  if (dev < 0 || dev >= static_cast<int>(rt->slots.size()) || !g->bind[dev] || rt->slots[dev]->remote)
    return fail(SF_EINVAL, "slot not bound locally");
  if (k0 < 0 || k0 >= static_cast<int>(g->parts.size()) || it0 < 0) return fail(SF_EINVAL, "bad cut");
  if (auto_target != SF_TARGET_HOST &&
      (auto_target < 0 || auto_target >= static_cast<int>(rt->slots.size()) || !g->bind[auto_target]))
    return fail(SF_EINVAL, "auto_target not bound");
  if (auto_target == SF_TARGET_HOST && !g->bind[dev]->host_staging)
    return fail(SF_EINVAL, "host tier needs host_staging");
  auto J = std::make_unique<Job>();
  J->id = static_cast<sf_job_id>(rt->jobs.size());
  J->g = g;
  J->dev = dev;
  J->iters = iters;
  J->auto_target = auto_target;
  J->home = dev;
  J->t_submit = now_ns();
  J->it = it0;
  J->k = k0;
  J->stamp_resume = it0 > 0 || k0 > 0;  // an adopted job: its first launch is the resume
  J->adopted_pending = J->stamp_resume;
  // DATASET contents are final once training starts: refresh padded-pitch copies
  for (auto& Bp : g->bind) {
    if (!Bp || Bp->remote) continue;
    for (auto& [t, sh] : Bp->shadow) {
      const Tensor& x = g->T[t];
      SF_CK(cudaSetDevice(rt->slots[Bp->slot]->cuda));
      SF_CK(cudaMemcpy2D(sh.first, static_cast<size_t>(sh.second) * 4, Bp->arena + x.offset,
                         static_cast<size_t>(x.cols) * 4, static_cast<size_t>(x.cols) * 4, x.rows,
                         cudaMemcpyDeviceToDevice));
    }
  }
  for (int i = 0; i < n_sched; ++i) {
    const sf_cut_request& c = sched[i];
    if (c.k < 0 || c.k >= static_cast<int>(g->parts.size()) || c.iter < 0)
      return fail(SF_EINVAL, "scheduled cut out of range");
    if (i > 0 && (c.iter < sched[i - 1].iter || (c.iter == sched[i - 1].iter && c.k <= sched[i - 1].k)))
      return fail(SF_EINVAL, "scheduled cuts must be strictly ascending");
    if (c.target != SF_TARGET_HOST &&
        (c.target < 0 || c.target >= static_cast<int>(rt->slots.size()) || !g->bind[c.target]))
      return fail(SF_EINVAL, "scheduled target not bound");
    J->sched.push_back(c);
  }
  if (sf_status s = ensure_events(rt, *J)) return s;
  if (g->feed) {
    Feed& F = *g->feed;
    if (F.shared) {
      if (it0 != 0 || k0 != 0) return fail(SF_EUNSUPPORTED, "shared-feed members start at iteration 0");
      if (F.member_jobs[g->feed_member] && F.member_jobs[g->feed_member]->state != SF_JOB_DONE)
        return fail(SF_EBUSY, "a job of this feed member is running");
    } else {
      // (re)start the pipeline at the job's first un-fed iteration; in-flight fills are stale
      ++F.gen;
      for (int s = 0; s < F.depth; ++s)
        if (F.slot_state[s] != 1) F.slot_state[s] = 0;
      F.next_iter = it0 + (k0 > 0 ? 1 : 0);
      F.inline_mode = rt->cfg.host_stage_inline != 0;
    }
    F.failed = false;
    F.active = true;
  }
  Job* jp = J.get();
  if (g->feed) g->feed->member_jobs[g->feed_member] = jp;
  rt->jobs.push_back(std::move(J));
  jp->driver = std::thread(driver_main, rt, jp);
  rt->cv.notify_all();  // lower-priority jobs on dev re-check their boundary gate
  *out = jp->id;
  return SF_OK;
}

sf_status sf_start_training(sf_runtime* rt, sf_graph_id gid, int32_t dev, int64_t iters,
                            int32_t auto_target, const sf_cut_request* sched, int32_t n_sched,
                            sf_job_id* out) {
  return start_job(rt, gid, dev, iters, auto_target, sched, n_sched, 0, 0, out);
}

sf_status sf_adopt_job(sf_runtime* rt, sf_graph_id gid, int32_t dev, int64_t iters, int64_t iter,
                       int32_t k, int32_t auto_target, sf_job_id* out) {
  return start_job(rt, gid, dev, iters, auto_target, nullptr, 0, iter, k, out);
}

sf_status sf_create_feed(sf_runtime* rt, const sf_feed_desc* d, sf_feed_id* out) {
  if (!rt || !d || !out || !d->fn || d->n < 1 || d->n > 8 || !d->bytes || d->depth < 0 || d->depth > 8)
    return fail(SF_EINVAL, "bad feed descriptor");
  std::lock_guard<std::mutex> lk(rt->m);
  auto F = std::make_unique<Feed>();
  F->id = static_cast<sf_feed_id>(rt->feeds.size());
  F->fn = d->fn;
  F->user = d->user;
  F->n = d->n;
  F->depth = d->depth ? d->depth : 2;
  F->shared = d->shared != 0;
  F->dev = d->dev;
  for (int i = 0; i < F->n; ++i) {
    if (d->bytes[i] == 0) return fail(SF_EINVAL, "empty fed tensor");
    F->off.push_back(F->stride);
    F->bytes.push_back(d->bytes[i]);
    F->stride += round_up(d->bytes[i], kAlign);
  }
  F->slot_iter.assign(F->depth, -1);
  F->slot_state.assign(F->depth, 0);
  F->consumed.assign(F->depth, 0);
  if (F->shared) {
    if (F->dev < 0 || F->dev >= static_cast<int>(rt->slots.size()) || rt->slots[F->dev]->remote)
      return fail(SF_EINVAL, "shared feed: dev is not a local slot");
    SF_CK(cudaSetDevice(rt->slots[F->dev]->cuda));
    SF_CK(cudaMalloc(&F->dbuf, F->stride * F->depth));
    SF_CK(cudaStreamCreateWithFlags(&F->st, cudaStreamNonBlocking));
    F->ev.assign(F->depth, nullptr);
    for (auto& e : F->ev) SF_CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  }
  SF_CK(cudaHostAlloc(&F->host, F->stride * F->depth, cudaHostAllocPortable));
  Feed* fp = F.get();
  rt->feeds.push_back(std::move(F));
  fp->stager = std::thread(stager_main, rt, fp);
  *out = fp->id;
  return SF_OK;
}

sf_status sf_attach_feed(sf_runtime* rt, sf_graph_id gid, sf_feed_id fid, const uint32_t* tids) {
  if (!rt || !tids) return fail(SF_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g) return fail(SF_EINVAL, "bad graph id");
  if (fid >= rt->feeds.size()) return fail(SF_EINVAL, "bad feed id");
  Feed& F = *rt->feeds[fid];
  if (g->feed) return fail(SF_ESTATE, "graph already has a feed");
  if (!F.shared && !F.members.empty()) return fail(SF_EBUSY, "a non-shared feed takes one graph");
  if (F.members.size() >= 32) return fail(SF_EINVAL, "at most 32 members per shared feed");
  for (int i = 0; i < F.n; ++i) {
    if (tids[i] >= g->T.size()) return fail(SF_EINVAL, "fed tensor id out of range");
    const Tensor& t = g->T[tids[i]];
    if ((t.kind != SF_INPUT && t.kind != SF_LABEL) || g->op_written[tids[i]])
      return fail(SF_EINVAL, "fed tensors are INPUT / LABEL tensors no op writes");
    if (t.nbytes != F.bytes[i]) return fail(SF_EINVAL, "fed tensor size differs from the feed's");
  }
  for (const auto& J : rt->jobs)
    if (J->g == g && J->state != SF_JOB_DONE && J->state != SF_JOB_FAILED)
      return fail(SF_ESTATE, "attach before starting the graph's jobs");
  g->feed = &F;
  g->feed_tids.assign(tids, tids + F.n);
  g->feed_member = static_cast<int>(F.members.size());
  F.members.push_back(g);
  F.member_jobs.push_back(nullptr);
  return SF_OK;
}

// Built-in host stage (sf.h: sf_stage_u8_normalize).  splitmix64 (Steele, Lea, Flood 2014):
// output n (1-based) of a generator seeded with s is fin(s + n * 0x9E3779B97F4A7C15).
static uint64_t splitmix64_out(uint64_t seed, uint64_t n) {
  uint64_t z = seed + n * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

int32_t sf_stage_u8_normalize(void* user, int64_t iter, void* const* dst, const uint64_t* bytes,
                              int32_t n) {
  const sf_u8_stage* u = static_cast<const sf_u8_stage*>(user);
  if (!u || !dst || n != 2 || u->batch <= 0 || u->cols <= 0 || u->img_w <= 0 || u->cols % u->img_w ||
      u->pool_rows < u->batch || u->pool_rows % u->batch || iter < 0)
    return -1;
  if (bytes[0] != static_cast<uint64_t>(u->batch) * u->cols * 4 || bytes[1] != static_cast<uint64_t>(u->batch) * 4)
    return -1;
  const int64_t b = iter % (u->pool_rows / u->batch);
  float* x = static_cast<float*>(dst[0]);
  int32_t* y = static_cast<int32_t*>(dst[1]);
  const int W = u->img_w, H = u->cols / u->img_w;
  for (int r = 0; r < u->batch; ++r) {
    const int64_t row = b * u->batch + r;
    const uint8_t* src = u->images + row * u->cols;
    float* xr = x + static_cast<int64_t>(r) * u->cols;
    if (splitmix64_out(u->seed, static_cast<uint64_t>(row) + 1) & 1) {
      for (int yy = 0; yy < H; ++yy)
        for (int xx = 0; xx < W; ++xx) xr[yy * W + xx] = static_cast<float>(src[yy * W + (W - 1 - xx)]) / 255.0f;
    } else {
      for (int c = 0; c < u->cols; ++c) xr[c] = static_cast<float>(src[c]) / 255.0f;
    }
    y[r] = u->labels[row];
  }
  return 0;
}

sf_status sf_export_arena(sf_runtime* rt, sf_graph_id gid, int32_t dev, sf_ipc_arena* out) {
  if (!rt || !out) return fail(SF_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g || dev < 0 || dev >= static_cast<int>(rt->slots.size()) || !g->bind[dev] || g->bind[dev]->remote)
    return fail(SF_EINVAL, "slot not bound locally");
  Binding& B = *g->bind[dev];
  SF_CK(cudaSetDevice(rt->slots[dev]->cuda));
  // driver entry point resolved at run time (no link-time libcuda dependency)
  using GetRange = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
  static GetRange get_range = nullptr;
  if (!get_range) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return fail(SF_ECUDA, "cuMemGetAddressRange entry point unavailable");
    get_range = reinterpret_cast<GetRange>(fn);
  }
  CUdeviceptr base = 0;
  size_t size = 0;
  if (get_range(&base, &size, reinterpret_cast<CUdeviceptr>(B.arena)) != CUDA_SUCCESS)
    return fail(SF_ECUDA, "cuMemGetAddressRange failed for the arena");
  cudaIpcMemHandle_t h;
  SF_CK(cudaIpcGetMemHandle(&h, reinterpret_cast<void*>(base)));
  std::memset(out, 0, sizeof(*out));
  std::memcpy(out->handle, &h, sizeof(h));
  out->offset = reinterpret_cast<uint64_t>(B.arena) - static_cast<uint64_t>(base);
  out->arena_bytes = g->arena_bytes;
  out->cuda_ordinal = rt->slots[dev]->cuda;
  return SF_OK;
}

sf_status sf_import_arena(sf_runtime* rt, sf_graph_id gid, int32_t slot, const sf_ipc_arena* a) {
  if (!rt || !a) return fail(SF_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* gp = get_graph(rt, gid);
  if (!gp || !gp->partitioned) return fail(SF_ESTATE, "graph not partitioned");
  Graph& g = *gp;
  if (slot < 0 || slot >= static_cast<int>(rt->slots.size()) || !rt->slots[slot]->remote)
    return fail(SF_EINVAL, "not a remote slot");
  if (g.bind[slot]) return fail(SF_ESTATE, "remote slot already mapped");
  if (a->arena_bytes != g.arena_bytes) return fail(SF_EINVAL, "arena layout mismatch");
  int local = -1;
  for (size_t o = 0; o < g.bind.size(); ++o)
    if (g.bind[o] && !g.bind[o]->remote) { local = static_cast<int>(o); break; }
  if (local < 0) return fail(SF_ESTATE, "bind a local slot before importing a remote arena");
  const int cuda = rt->slots[local]->cuda;
  SF_CK(cudaSetDevice(cuda));
  cudaIpcMemHandle_t h;
  std::memcpy(&h, a->handle, sizeof(h));
  void* p = nullptr;
  SF_CK(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
  auto b = std::make_unique<Binding>();
  b->slot = slot;
  b->remote = true;
  b->ipc_base = p;
  b->ipc_device = cuda;
  b->arena = static_cast<uint8_t*>(p) + a->offset;
  g.bind[slot] = std::move(b);
  for (size_t o = 0; o < g.bind.size(); ++o) {
    if (static_cast<int>(o) == slot || !g.bind[o] || g.bind[o]->remote) continue;
    if (sf_status s = build_peer_lists(rt, g, *g.bind[o], *g.bind[slot])) return s;
  }
  return SF_OK;
}

sf_status sf_preempt(sf_runtime* rt, sf_job_id jid, int32_t target, sf_cut_info* out) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::unique_lock<std::mutex> lk(rt->m);
  Job* J = get_job(rt, jid);
  if (!J) return fail(SF_EINVAL, "bad job id");
  if (J->state == SF_JOB_MIGRATING) return fail(SF_EBUSY, "migration in flight");
  if (J->state != SF_JOB_RUNNING || J->preempt_req) return fail(SF_ESTATE, "job not running");
  if (target == J->dev) return fail(SF_EINVAL, "target is the current device");
  if (target == SF_TARGET_HOST) {
    if (!J->g->bind[J->dev]->host_staging) return fail(SF_EINVAL, "no host staging bound");
  } else if (target < 0 || target >= static_cast<int>(rt->slots.size()) || !J->g->bind[target]) {
    return fail(SF_EINVAL, "target slot not bound");
  }
  J->cut_ready = false;
  J->preempt_req = true;
  J->preempt_park = true;
  J->preempt_target = target;
  J->t_req = now_ns();
  rt->cv.notify_all();
  rt->cv.wait(lk, [&] { return J->cut_ready || J->state == SF_JOB_DONE || J->state == SF_JOB_FAILED; });
  if (!J->cut_ready) return fail(SF_ESTATE, "job finished before reaching a boundary: " + J->error);
  rt->cv.wait(lk, [&] { return J->mig_enqueued || J->state == SF_JOB_FAILED; });
  if (J->state == SF_JOB_FAILED) return fail(SF_ECUDA, J->error);
  if (out) *out = J->cut;
  return SF_OK;
}

sf_status sf_resume(sf_runtime* rt, sf_job_id jid, int32_t dev) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::lock_guard<std::mutex> lk(rt->m);
  Job* J = get_job(rt, jid);
  if (!J) return fail(SF_EINVAL, "bad job id");
  if (J->state != SF_JOB_PREEMPTED) return fail(SF_ESTATE, "job not preempted");
  if (dev < 0 || dev >= static_cast<int>(rt->slots.size()) || !J->g->bind[dev])
    return fail(SF_EINVAL, "slot not bound");
  if (J->cut.dst_dev != SF_TARGET_HOST && dev != J->cut.dst_dev)
    return fail(SF_EINVAL, "peer-migrated job resumes on its migration target");
  J->resume_req = true;
  J->resume_dev = dev;
  J->state = SF_JOB_RUNNING;  // visible to the caller at once; the driver continues
  rt->cv.notify_all();
  return SF_OK;
}

sf_status sf_job_query(sf_runtime* rt, sf_job_id jid, sf_job_info* out) {
  if (!rt || !out) return fail(SF_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(rt->m);
  Job* J = get_job(rt, jid);
  if (!J) return fail(SF_EINVAL, "bad job id");
  out->state = J->state;
  out->dev = J->dev;
  out->iter = J->it;
  out->k = J->k;
  out->n_preemptions = J->n_preempt;
  out->migrated_bytes = J->migrated;
  out->last_pack_us = J->pack_us;
  out->last_xfer_us = J->xfer_us;
  out->last_unpack_us = J->unpack_us;
  out->last_stop_ns = J->last_stop;
  out->last_resume_ns = J->last_resume;
  out->n_reparks = J->n_repark;
  out->submit_ns = J->t_submit;
  out->priority = J->g->priority;
  out->home = J->home;
  if (J->state == SF_JOB_FAILED) return fail(SF_ECUDA, J->error);
  return SF_OK;
}

sf_status sf_read_tensor(sf_runtime* rt, sf_job_id jid, uint32_t tid, void* host_dst, size_t n) {
  if (!rt || !host_dst) return fail(SF_EINVAL, "null argument");
  const uint8_t* src = nullptr;
  cudaStream_t st = nullptr;
  int cuda = 0;
  {
    std::lock_guard<std::mutex> lk(rt->m);
    Job* J = get_job(rt, jid);
    if (!J) return fail(SF_EINVAL, "bad job id");
    Graph& g = *J->g;
    if (tid >= g.T.size() || n != g.T[tid].nbytes) return fail(SF_EINVAL, "bad tensor id / size");
    if (J->state == SF_JOB_MIGRATING || J->state == SF_JOB_STOPPING || J->state == SF_JOB_MIGRATED_OUT ||
        (J->state == SF_JOB_PREEMPTED && J->cut.dst_dev == SF_TARGET_HOST))
      return fail(SF_EBUSY, "the job's state is in transit or parked in host memory");
    if (J->dev < 0 || !g.bind[J->dev] || g.bind[J->dev]->remote) return fail(SF_ESTATE, "job not on a local slot");
    Slot& S = *rt->slots[J->dev];
    src = g.bind[J->dev]->arena + g.T[tid].offset;
    st = S.s_train;
    cuda = S.cuda;
  }
  SF_CK(cudaSetDevice(cuda));
  SF_CK(cudaMemcpyAsync(host_dst, src, n, cudaMemcpyDeviceToHost, st));
  SF_CK(cudaStreamSynchronize(st));
  return SF_OK;
}

sf_status sf_wait_job(sf_runtime* rt, sf_job_id jid, int64_t timeout_ns) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::unique_lock<std::mutex> lk(rt->m);
  Job* J = get_job(rt, jid);
  if (!J) return fail(SF_EINVAL, "bad job id");
  auto done = [&] {
    return J->state == SF_JOB_DONE || J->state == SF_JOB_FAILED || J->state == SF_JOB_MIGRATED_OUT;
  };
  if (timeout_ns < 0) rt->cv.wait(lk, done);
  else if (!rt->cv.wait_for(lk, std::chrono::nanoseconds(timeout_ns), done))
    return fail(SF_ETIMEOUT, "job still running");
  if (J->state == SF_JOB_FAILED) return fail(SF_ECUDA, J->error);
  return SF_OK;
}

sf_status sf_stop_job(sf_runtime* rt, sf_job_id jid) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::lock_guard<std::mutex> lk(rt->m);
  Job* J = get_job(rt, jid);
  if (!J) return fail(SF_EINVAL, "bad job id");
  J->stop_req = true;
  rt->cv.notify_all();
  return SF_OK;
}

sf_status sf_submit_inference(sf_runtime* rt, sf_graph_id gid, int32_t dev, const void* in,
                              void* out, uint64_t arrival_ns, sf_req_id* req) {
  if (!rt || !in || !out || !req) return fail(SF_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g || !g->partitioned) return fail(SF_ESTATE, "graph not partitioned");
  if (dev < 0 || dev >= static_cast<int>(rt->slots.size()) || !g->bind[dev] || rt->slots[dev]->remote)
    return fail(SF_EINVAL, "slot not bound locally");
  if (g->input_tid < 0 || g->output_tid < 0) return fail(SF_EINVAL, "graph has no INPUT/OUTPUT");
  auto r = std::make_unique<Request>();
  r->id = rt->next_req++;
  r->g = g;
  r->dev = dev;
  r->in = in;
  r->out = out;
  r->arrival = arrival_ns ? arrival_ns : now_ns();
  Request* rp = r.get();
  rt->reqs.emplace(r->id, std::move(r));
  rt->slots[dev]->q.push_back(rp);
  rt->slots[dev]->qn.fetch_add(1);
  *req = rp->id;
  rt->cv.notify_all();
  return SF_OK;
}

sf_status sf_wait(sf_runtime* rt, sf_req_id id, int64_t timeout_ns, sf_timing* t) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::unique_lock<std::mutex> lk(rt->m);
  auto it = rt->reqs.find(id);
  if (it == rt->reqs.end()) return fail(SF_EINVAL, "unknown request");
  Request* r = it->second.get();
  auto done = [&] { return r->done; };
  if (timeout_ns < 0) rt->cv.wait(lk, done);
  else if (!rt->cv.wait_for(lk, std::chrono::nanoseconds(timeout_ns), done))
    return fail(SF_ETIMEOUT, "request pending");
  if (t) {
    t->arrival_ns = r->arrival;
    t->start_ns = r->start;
    t->end_ns = r->end;
    t->dev = r->dev;
    t->preempted_job = r->preempted_job;
    t->cut_iter = r->cut_iter;
    t->cut_k = r->cut_k;
    t->device_us = r->device_us;
    t->launch_us = r->launch_us;
    t->dispatch_us = r->dispatch_us;
  }
  std::string err = r->error;
  rt->reqs.erase(it);
  if (!err.empty()) return fail(SF_ECUDA, err);
  return SF_OK;
}

sf_status sf_get_trace(sf_runtime* rt, sf_trace_event* buf, size_t cap, size_t* n_out) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::lock_guard<std::mutex> lk(rt->m);
  const size_t n = std::min(cap, rt->trace.size());
  if (buf) {
    std::copy(rt->trace.begin(), rt->trace.begin() + n, buf);
    // device intervals through ONE mapping (the slot's anchors as of now) for every event read
    // together: their order is the GPU's order (reading Q37); events without a device-timeline
    // position keep the value mapped at completion
    for (size_t i = 0; i < n && i < rt->trace_D.size(); ++i) {
      sf_trace_event& e = buf[i];
      if (e.kind != SF_EV_TRAIN && e.kind != SF_EV_INFER) continue;
      if (e.dev < 0 || static_cast<size_t>(e.dev) >= rt->slots.size() || !rt->slots[e.dev]) continue;
      Slot& S = *rt->slots[e.dev];
      const auto [D0, D1] = rt->trace_D[i];
      if (std::isnan(D0) || std::isnan(D1)) continue;
      const uint64_t m0 = dev_D_to_host(S, D0), m1 = dev_D_to_host(S, D1);
      if (m0 && m1) { e.d0_ns = m0; e.d1_ns = m1; }
    }
  }
  if (n_out) *n_out = buf ? n : rt->trace.size();
  return SF_OK;
}

// ---- direct kernel entry points --------------------------------------------------------
static cudaStream_t as_stream(void* s) { return static_cast<cudaStream_t>(s); }

sf_status sf_op_mtcopy(const sf_copy_desc* descs, int32_t n, int64_t patch_iter, void* stream) {
  if (n < 0 || (n > 0 && !descs)) return fail(SF_EINVAL, "descs");
  if (n == 0) return SF_OK;
  std::vector<sfk::DCopy> d;
  uint64_t chunks = 0;
  for (int i = 0; i < n; ++i) {
    const sf_copy_desc& s = descs[i];
    if (s.span < s.nbytes || s.span % 16 || s.nbytes % 4 ||
        reinterpret_cast<uintptr_t>(s.src) % 16 || reinterpret_cast<uintptr_t>(s.dst) % 16)
      return fail(SF_EINVAL, "descriptor " + std::to_string(i) + ": alignment / span");
    d.push_back({static_cast<const uint8_t*>(s.src), static_cast<uint8_t*>(s.dst), s.nbytes, chunks});
    chunks += s.span / 16;
  }
  sfk::DCopy sent{};
  sent.chunk_begin = chunks;
  d.push_back(sent);
  cudaStream_t st = as_stream(stream);
  void* dd = nullptr;
  SF_CK(cudaMallocAsync(&dd, d.size() * sizeof(sfk::DCopy), st));
  SF_CK(cudaMemcpyAsync(dd, d.data(), d.size() * sizeof(sfk::DCopy), cudaMemcpyHostToDevice, st));
  SF_CK(sfk::launch_mtcopy(static_cast<sfk::DCopy*>(dd), n, chunks, patch_iter, st));
  SF_CK(cudaFreeAsync(dd, st));
  SF_CK(cudaStreamSynchronize(st));  // the host descriptor array is released on return
  return SF_OK;
}

static sf_status op_gemm(const float* A, const float* B, float* C, int32_t M, int32_t N, int32_t K,
                         int32_t lda, int32_t ldb, int32_t ldc, int32_t flags, const float* b1,
                         const float* b2, const float* b3, bool relu, void* stream) {
  if (!A || !B || !C || M <= 0 || N <= 0 || K <= 0) return fail(SF_EINVAL, "gemm args");
  if (!b1 && (b2 || b3)) return fail(SF_EINVAL, "gemm bias args");
  sfk::GemmArgs ga{A, B, C, M, N, K, lda, ldb, ldc, (flags & SF_GEMM_TA) != 0,
                   (flags & SF_GEMM_TB) != 0, (flags & SF_GEMM_ACC) != 0, nullptr, nullptr};
  const bool epi = b1 || relu;
  const bool fuse = epi && (sfk::gemm_can_fuse_bias(M, N, K, ga.ta, ga.tb, ldb) || sfk::gemv_rows_eligible(ga));
  if (fuse) {
    ga.bias[0] = b1; ga.bias[1] = b2; ga.bias[2] = b3;
    ga.relu = relu;
  }
  cudaStream_t st = as_stream(stream);
  const uint64_t wsf = sfk::gemm_workspace_floats(M, N, K, ga.ta, ga.tb);
  const uint64_t cs = sfk::gemm_counter_slots(M, N, K, ga.ta, ga.tb);
  if (wsf) {
    // split-K workspace + reduction counters cached per (device, stream) and grown on demand
    // (stream-ordered free of the old buffers); the counters reset themselves after every
    // reduction, so they are zeroed once, at allocation
    struct OpWs { float* ws = nullptr; unsigned* cnt = nullptr; uint64_t wsf = 0, cs = 0; };
    static std::mutex m;
    static std::map<std::pair<int, cudaStream_t>, OpWs> cache;
    int dev = 0;
    SF_CK(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> g(m);
    OpWs& w = cache[{dev, st}];
    if (w.wsf < wsf || w.cs < cs) {
      if (w.ws) { SF_CK(cudaFreeAsync(w.ws, st)); SF_CK(cudaFreeAsync(w.cnt, st)); }
      w.wsf = std::max(w.wsf, wsf);
      w.cs = std::max(w.cs, cs);
      SF_CK(cudaMallocAsync(reinterpret_cast<void**>(&w.ws), w.wsf * 4, st));
      SF_CK(cudaMallocAsync(reinterpret_cast<void**>(&w.cnt), w.cs * 4, st));
      SF_CK(cudaMemsetAsync(w.cnt, 0, w.cs * 4, st));
    }
    ga.ws = w.ws;
    ga.counters = w.cnt;
    SF_CK(sfk::launch_gemm(ga, st));
  } else {
    SF_CK(sfk::launch_gemm(ga, st));
  }
  if (epi && !fuse) {
    if (ldc != N) return fail(SF_EINVAL, "unfused gemm epilogue needs ldc == N");
    SF_CK(sfk::launch_bias_act(C, b1, b2, b3, C, M, N, relu, st));
  }
  return SF_OK;
}

sf_status sf_op_gemm(const float* A, const float* B, float* C, int32_t M, int32_t N, int32_t K,
                     int32_t lda, int32_t ldb, int32_t ldc, int32_t flags, void* stream) {
  return op_gemm(A, B, C, M, N, K, lda, ldb, ldc, flags, nullptr, nullptr, nullptr, false, stream);
}

sf_status sf_probe_migration(sf_runtime* rt, sf_graph_id gid, int32_t dev, int32_t k, int32_t l2,
                             sf_migration_probe* out) {
  if (!rt || !out || l2 < 0 || l2 > 2) return fail(SF_EINVAL, "bad argument");
  Graph* g = nullptr;
  Binding* B = nullptr;
  Slot* S = nullptr;
  {
    std::lock_guard<std::mutex> lk(rt->m);
    g = get_graph(rt, gid);
    if (!g || !g->partitioned || k < 0 || k >= static_cast<int>(g->parts.size()))
      return fail(SF_EINVAL, "bad graph / cut");
    if (dev < 0 || dev >= static_cast<int>(rt->slots.size()) || !g->bind[dev] || g->bind[dev]->remote)
      return fail(SF_EINVAL, "slot not bound locally");
    B = g->bind[dev].get();
    if (!B->staging) return fail(SF_EINVAL, "no device staging bound");
    for (const auto& J : rt->jobs)
      if (J->g == g && (J->state == SF_JOB_RUNNING || J->state == SF_JOB_STOPPING ||
                        J->state == SF_JOB_MIGRATING))
        return fail(SF_EBUSY, "a job of this graph is running");
    S = rt->slots[dev].get();
  }
  SF_CK(cudaSetDevice(S->cuda));
  int l2size = 0;
  SF_CK(cudaDeviceGetAttribute(&l2size, cudaDevAttrL2CacheSize, S->cuda));
  const uint64_t fb = round_up(2ull * static_cast<uint64_t>(l2size), 4096);
  void* scratch = nullptr;
  if (l2) SF_CK(cudaMalloc(&scratch, fb));
  double us[2] = {0, 0};
  for (int w = 0; w < 2; ++w) {
    const CopyList& L = w == 0 ? B->pack[k] : B->unpack[k];
    cudaError_t e = l2 == 1 ? sfk::launch_read_flush(scratch, fb, S->s_mig)
                  : l2 == 2 ? sfk::launch_fill(scratch, fb, 0x5A, S->s_mig) : cudaSuccess;
    if (e == cudaSuccess) e = tstamp_reset(S->tstamp, S->s_mig);
    if (e == cudaSuccess) e = sfk::launch_mtcopy(L.d, L.n, L.total_chunks, w == 0 ? 0 : -1, S->s_mig, S->tstamp);
    if (e == cudaSuccess) e = cudaStreamSynchronize(S->s_mig);
    if (e != cudaSuccess) {
      if (scratch) cudaFree(scratch);
      return fail(SF_ECUDA, std::string("probe: ") + cudaGetErrorString(e));
    }
    us[w] = tstamp_us(S->tstamp);
  }
  if (scratch) SF_CK(cudaFree(scratch));
  out->pack_us = us[0];
  out->unpack_us = us[1];
  out->live_bytes = g->live_bytes[k];
  out->staging_bytes = g->staging_total[k];
  return SF_OK;
}

sf_status sf_probe_peer(sf_runtime* rt, sf_graph_id gid, int32_t src, int32_t dst, int32_t k,
                        int32_t engine, double* us, uint64_t* bytes_moved) {
  if (!rt || !us || engine < 0 || engine > 3) return fail(SF_EINVAL, "bad argument");
  Graph* g = nullptr;
  Binding *B = nullptr, *D = nullptr;
  Slot* S = nullptr;
  {
    std::lock_guard<std::mutex> lk(rt->m);
    g = get_graph(rt, gid);
    if (!g || !g->partitioned || k < 0 || k >= static_cast<int>(g->parts.size()))
      return fail(SF_EINVAL, "bad graph / cut");
    const int ns = static_cast<int>(rt->slots.size());
    if (src < 0 || src >= ns || dst < 0 || dst >= ns || src == dst || !g->bind[src] || g->bind[src]->remote ||
        !g->bind[dst])
      return fail(SF_EINVAL, "bad slots");
    B = g->bind[src].get();
    D = g->bind[dst].get();
    if (!B->peer.count(dst)) return fail(SF_EINVAL, "no peer list to dst");
    for (const auto& J : rt->jobs)
      if (J->g == g && (J->state == SF_JOB_RUNNING || J->state == SF_JOB_STOPPING ||
                        J->state == SF_JOB_MIGRATING))
        return fail(SF_EBUSY, "a job of this graph is running");
    S = rt->slots[src].get();
  }
  SF_CK(cudaSetDevice(S->cuda));
  cudaEvent_t e0, e1;
  SF_CK(cudaEventCreate(&e0));
  SF_CK(cudaEventCreate(&e1));
  uint64_t moved = g->live_bytes[k];
  cudaError_t e = tstamp_reset(S->tstamp, S->s_mig);
  if (e == cudaSuccess) e = cudaEventRecord(e0, S->s_mig);
  if (e == cudaSuccess) {
    if (engine == 0) {
      const CopyList& L = B->peer[dst][k];
      e = sfk::launch_mtcopy(L.d, L.n, L.total_chunks, -1, S->s_mig, S->tstamp);
    } else if (engine == 1) {
      Job none;
      e = ce_segments(none, *S, src, cut_segments(*g, k, B->arena, D->arena, 2), S->s_mig, false);
    } else if (engine == 2) {
      for (const Seg& sg : cut_segments(*g, k, B->arena, D->arena, 2))
        if ((e = cudaMemcpyAsync(sg.dst, sg.src, sg.n, cudaMemcpyDefault, S->s_mig)) != cudaSuccess) break;
    } else {
      uint64_t lo = ~0ull, hi = 0;
      for (uint32_t t : g->live[k]) {
        lo = std::min(lo, g->T[t].offset);
        hi = std::max(hi, g->T[t].offset + g->T[t].nbytes);
      }
      moved = hi > lo ? hi - lo : 0;
      if (moved) e = cudaMemcpyAsync(D->arena + lo, B->arena + lo, moved, cudaMemcpyDefault, S->s_mig);
    }
  }
  if (e == cudaSuccess) e = cudaEventRecord(e1, S->s_mig);
  if (e == cudaSuccess) e = cudaStreamSynchronize(S->s_mig);
  double t = -1.0;
  if (e == cudaSuccess) {
    t = engine == 0 ? tstamp_us(S->tstamp) : -1.0;
    if (t < 0) t = elapsed_us(e0, e1);
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (e != cudaSuccess) return fail(SF_ECUDA, std::string("probe peer: ") + cudaGetErrorString(e));
  *us = t;
  if (bytes_moved) *bytes_moved = moved;
  return SF_OK;
}

sf_status sf_refresh_constants(sf_runtime* rt, sf_graph_id gid, int32_t dev) {
  if (!rt) return fail(SF_EINVAL, "null runtime");
  std::lock_guard<std::mutex> lk(rt->m);
  Graph* g = get_graph(rt, gid);
  if (!g || dev < 0 || dev >= static_cast<int>(rt->slots.size()) || !g->bind[dev] || g->bind[dev]->remote)
    return fail(SF_EINVAL, "slot not bound locally");
  Binding& B = *g->bind[dev];
  Slot& S = *rt->slots[dev];
  SF_CK(cudaSetDevice(S.cuda));
  // re-laid out now, ordered before any later request on the request stream
  layout_blocked(*g, B, S.s_infer);
  SF_CK(cudaStreamSynchronize(S.s_infer));
  B.blocked_ready = true;
  if (infer_graph_mode()) {
    static const bool use_pdl = !(std::getenv("SF_PDL") && std::getenv("SF_PDL")[0] == '0');
    build_req_graph(*g, B, use_pdl);
  }
  return SF_OK;
}

sf_status sf_slot_query(sf_runtime* rt, int32_t slot, sf_slot_info* out) {
  if (!rt || !out) return fail(SF_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(rt->m);
  if (slot < 0 || slot >= static_cast<int>(rt->slots.size())) return fail(SF_EINVAL, "bad slot");
  Slot& S = *rt->slots[slot];
  std::memset(out, 0, sizeof(*out));
  out->owner = S.owner.load();
  out->queued = static_cast<int32_t>(S.q.size());
  out->gate_held = S.gate_held ? 1 : 0;
  out->gate_value = S.gate ? S.gate[0] : 0;
  out->gate_arrived = S.gate ? S.gate[16] : 0;
  out->next_ticket = S.next_ticket;
  out->gate_valve = static_cast<uint32_t>(S.gate_valve);
  return SF_OK;
}

sf_status sf_last_gemm_path(sf_gemm_path* out) {
  if (!out) return fail(SF_EINVAL, "null argument");
  const sfk::GemmPath p = sfk::last_gemm_path();
  out->kind = p.kind;
  out->bn = p.bn;
  out->splits = p.splits;
  out->a_mn = p.a_mn;
  out->b_mn = p.b_mn;
  out->pad = 0;
  return SF_OK;
}

sf_status sf_debug_chain_trace(void* dev_buf) {
  sfk::set_chain_trace(dev_buf);
  return SF_OK;
}

sf_status sf_op_mlp_chain(const float* x, int32_t M, int32_t n_layers, const int32_t* widths,
                          const float* const* W, const float* const* b, const int32_t* relu,
                          float* const* h, float* probs, void* stream) {
  if (!x || !widths || !W || !h || n_layers < 1) return fail(SF_EINVAL, "mlp_chain args");
  if (n_layers > sfk::kChainMaxLayers) return fail(SF_EUNSUPPORTED, "mlp_chain: too many layers");
  sfk::ChainArgs a;
  a.M = M;
  a.n_layers = n_layers;
  for (int l = 0; l < n_layers; ++l) {
    sfk::ChainLayerArgs& L = a.layer[l];
    L = sfk::ChainLayerArgs{};
    L.K = widths[l];
    L.N = widths[l + 1];
    L.W = W[l]; L.ldw = L.N;
    L.x = l == 0 ? x : h[l - 1]; L.ldx = L.K;
    L.y = h[l]; L.ldy = L.N;
    L.b[0] = b ? b[l] : nullptr;
    L.relu = relu && relu[l];
  }
  if (probs) {
    a.softmax = true;
    a.sm_out = probs;
    a.sm_n = widths[n_layers];
    a.sm_ldi = a.sm_ldo = widths[n_layers];
  }
  if (!sfk::chain_eligible(a)) return fail(SF_EUNSUPPORTED, "mlp_chain: shape outside the fused kernel");
  cudaStream_t st = as_stream(stream);
  const uint64_t wf = sfk::chain_ws_floats(a), cs = sfk::chain_counter_slots(a);
  void *ws = nullptr, *cnt = nullptr, *w0t = nullptr;
  SF_CK(cudaMallocAsync(&ws, std::max<uint64_t>(wf, 4) * 4, st));
  SF_CK(cudaMallocAsync(&cnt, cs * 4, st));
  SF_CK(cudaMallocAsync(&w0t, sfk::chain_w0t_floats(widths[0], widths[1]) * 4, st));
  SF_CK(cudaMemsetAsync(cnt, 0, cs * 4, st));
  SF_CK(sfk::launch_chain_w0t_layout(W[0], widths[1], widths[0], widths[1], static_cast<float*>(w0t), st));
  a.ws = static_cast<float*>(ws);
  a.counters = static_cast<unsigned*>(cnt);
  a.w0t = static_cast<float*>(w0t);
  SF_CK(sfk::launch_chain(a, st));
  SF_CK(cudaFreeAsync(ws, st));
  SF_CK(cudaFreeAsync(cnt, st));
  SF_CK(cudaFreeAsync(w0t, st));
  return SF_OK;
}

sf_status sf_op_gemm_bias_act(const float* A, const float* B, float* C, int32_t M, int32_t N,
                              int32_t K, int32_t lda, int32_t ldb, int32_t ldc, int32_t flags,
                              const float* b1, const float* b2, const float* b3, int32_t relu,
                              void* stream) {
  if (!b1) return fail(SF_EINVAL, "gemm_bias_act needs b1");
  return op_gemm(A, B, C, M, N, K, lda, ldb, ldc, flags, b1, b2, b3, relu != 0, stream);
}

sf_status sf_op_bias_act(const float* z, const float* b1, const float* b2, const float* b3,
                         float* h, int32_t rows, int32_t cols, int32_t act, void* stream) {
  if (!z || !b1 || !h) return fail(SF_EINVAL, "bias_act args");
  if (act < 0 || act > SF_ACT_GELU) return fail(SF_EINVAL, "bias_act: act must be 0, RELU or GELU");
  SF_CK(sfk::launch_bias_act(z, b1, b2, b3, h, rows, cols, act, as_stream(stream)));
  return SF_OK;
}

static sf_status colsum_common(const float* x, const float* mask, float* dz, float* s, int rows,
                               int cols, cudaStream_t st, int mode = 1) {
  const uint64_t wsf = sfk::colsum_ws_floats(rows, cols);
  const uint64_t cs = sfk::colsum_counter_slots(rows, cols);
  void* ws = nullptr;
  void* cnt = nullptr;
  if (wsf) {
    SF_CK(cudaMallocAsync(&ws, wsf * 4, st));
    SF_CK(cudaMallocAsync(&cnt, cs * 4, st));
    SF_CK(cudaMemsetAsync(cnt, 0, cs * 4, st));
  }
  SF_CK(sfk::launch_colsum(x, mask, dz, s, rows, cols, static_cast<float*>(ws),
                           static_cast<unsigned*>(cnt), st, mode));
  if (ws) {
    SF_CK(cudaFreeAsync(ws, st));
    SF_CK(cudaFreeAsync(cnt, st));
  }
  return SF_OK;
}

sf_status sf_op_bias_act_bwd(const float* dh, const float* h, float* dz, float* db, int32_t rows,
                             int32_t cols, void* stream) {
  if (!dh || !h || !dz || !db) return fail(SF_EINVAL, "bias_act_bwd args");
  return colsum_common(dh, h, dz, db, rows, cols, as_stream(stream));
}

sf_status sf_op_gelu_bwd(const float* dh, const float* u, float* dz, float* db, int32_t rows,
                         int32_t cols, void* stream) {
  if (!dh || !u || !dz || !db) return fail(SF_EINVAL, "gelu_bwd args");
  return colsum_common(dh, u, dz, db, rows, cols, as_stream(stream), 2);
}

sf_status sf_op_colsum(const float* x, float* s, int32_t rows, int32_t cols, void* stream) {
  if (!x || !s) return fail(SF_EINVAL, "colsum args");
  return colsum_common(x, nullptr, nullptr, s, rows, cols, as_stream(stream));
}

sf_status sf_op_softmax_ce(const float* logits, const int32_t* labels, float* loss, float* dlogits,
                           int32_t rows, int32_t cols, void* stream) {
  if (!logits || !labels || !loss || !dlogits || rows <= 0 || cols <= 0)
    return fail(SF_EINVAL, "softmax_ce args");
  cudaStream_t st = as_stream(stream);
  void *ws = nullptr, *cnt = nullptr;
  SF_CK(cudaMallocAsync(&ws, sfk::softmax_ce_ws_floats(rows) * 4, st));
  SF_CK(cudaMallocAsync(&cnt, 16, st));
  SF_CK(cudaMemsetAsync(cnt, 0, 16, st));
  SF_CK(sfk::launch_softmax_ce(logits, labels, loss, dlogits, rows, cols, static_cast<float*>(ws),
                               static_cast<unsigned*>(cnt), st));
  SF_CK(cudaFreeAsync(ws, st));
  SF_CK(cudaFreeAsync(cnt, st));
  return SF_OK;
}

sf_status sf_op_softmax(const float* logits, float* probs, int32_t rows, int32_t cols, void* stream) {
  if (!logits || !probs) return fail(SF_EINVAL, "softmax args");
  SF_CK(sfk::launch_softmax(logits, probs, rows, cols, as_stream(stream)));
  return SF_OK;
}

static bool al16(const void* p) { return reinterpret_cast<uintptr_t>(p) % 16 == 0; }

sf_status sf_op_sgd_mom(float* w, float* a, const float* g, int64_t n, float lr, float mu,
                        void* stream) {
  if (!w || !a || !g || n < 0 || !al16(w) || !al16(a) || !al16(g))
    return fail(SF_EINVAL, "sgd args (16-B aligned pointers)");
  cudaStream_t st = as_stream(stream);
  sfk::SgdDesc d[2] = {{w, a, g, static_cast<uint64_t>(n), lr, mu, 0}, {}};
  d[1].begin = (static_cast<uint64_t>(n) + 3) / 4;
  void* dd = nullptr;
  SF_CK(cudaMallocAsync(&dd, sizeof(d), st));
  SF_CK(cudaMemcpyAsync(dd, d, sizeof(d), cudaMemcpyHostToDevice, st));
  SF_CK(sfk::launch_sgd(static_cast<sfk::SgdDesc*>(dd), 1, d[1].begin, st));
  SF_CK(cudaFreeAsync(dd, st));
  SF_CK(cudaStreamSynchronize(st));
  return SF_OK;
}

sf_status sf_op_adam(float* w, float* m, float* v, const float* g, const int32_t* step, int64_t n,
                     float lr, float beta1, float beta2, float eps, void* stream) {
  if (!w || !m || !v || !g || !step || n < 0 || !al16(w) || !al16(m) || !al16(v) || !al16(g))
    return fail(SF_EINVAL, "adam args (16-B aligned pointers)");
  cudaStream_t st = as_stream(stream);
  sfk::AdamDesc d[2] = {{w, m, v, g, static_cast<uint64_t>(n), lr, beta1, beta2, eps, 0}, {}};
  d[1].begin = (static_cast<uint64_t>(n) + 3) / 4;
  void* dd = nullptr;
  SF_CK(cudaMallocAsync(&dd, sizeof(d), st));
  SF_CK(cudaMemcpyAsync(dd, d, sizeof(d), cudaMemcpyHostToDevice, st));
  SF_CK(sfk::launch_adam(static_cast<sfk::AdamDesc*>(dd), 1, d[1].begin, step, st));
  SF_CK(cudaFreeAsync(dd, st));
  SF_CK(cudaStreamSynchronize(st));
  return SF_OK;
}

sf_status sf_op_fill(void* dst, uint64_t n, int32_t value, void* stream) {
  if (!dst) return fail(SF_EINVAL, "fill args");
  SF_CK(sfk::launch_fill(dst, n, static_cast<uint8_t>(value), as_stream(stream)));
  return SF_OK;
}

}  // extern "C"
