/*
 * sf.h — C ABI of the SwitchFlow-on-B200 subgraph-preemption runtime.
 *
 * Method: SwitchFlow, "Preemptive Multitasking for Deep Learning" (Wu et al.,
 * Middleware '21), /root/reference/PAPER.md.  The ABI follows the paper's problem
 * statement: jobs are static computation graphs (section 2) submitted
 * with a priority (section 4); the session is partitioned into
 * subgraphs run by executors (section 2.1) and one executor version is
 * built per device (section 3.2); a high-priority job "is allowed to
 * start immediately after submission" (section 3.4); the preemptee is
 * suspended, its graph re-pointed at another device, its persistent state copied
 * asynchronously, and it resumes with no work lost (section 3.3); no two
 * models' GPU executors co-run on one GPU (section 3.4).
 *
 * B200 design: a preemption cuts the job at its next subgraph boundary and
 * migrates the live set L_k (variables, optimizer slots, in-flight activations) — to a
 * peer B200 over NVLink with a fused peer-store kernel, or to pinned host memory
 * (pack kernel + PCIe) — and resumes the pre-built CUDA-graph version of S_k there.
 *
 * Conventions (all entry points):
 *  - every call returns sf_status; SF_OK == 0, errors < 0; no exception crosses the ABI;
 *    the message of the last error on the calling thread is in sf_last_error();
 *  - "device pointer" = CUDA global memory of the stated device (or a peer mapping);
 *    "host pointer" = ordinary host memory; "pinned" = page-locked (cudaHostAlloc /
 *    torch pin_memory) host memory;
 *  - memory passed in (arenas, staging, request buffers, op operands) is CALLER-OWNED
 *    and must stay valid until the call that uses it completes (for sf_bind: until
 *    sf_destroy); runtime-owned memory (descriptor lists, CUDA graphs, workspaces,
 *    events, threads) is freed only by sf_destroy;
 *  - tensors are 2-D row-major; fp32 (SF_F32) or int32 (SF_I32); arenas place every
 *    tensor at a 256-byte aligned offset, identical on every device;
 *  - all sf_* calls are thread-safe.  sf_op_* kernel entry points are asynchronous on
 *    the given stream (cudaStream_t passed as void*, NULL = legacy default stream).
 */
#ifndef SF_H_
#define SF_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SF_ABI_VERSION 1

typedef int32_t sf_status;
#define SF_OK 0
#define SF_EINVAL (-1)       /* bad argument / malformed graph */
#define SF_ENOMEM (-2)       /* device budget exceeded or allocation failed */
#define SF_ESTATE (-3)       /* call not valid in the object's current state */
#define SF_EBUSY (-4)        /* a migration of this job is already in flight */
#define SF_ECUDA (-5)        /* CUDA error; text in sf_last_error() */
#define SF_ETIMEOUT (-6)
#define SF_EUNSUPPORTED (-7) /* op outside the fixed op set, or dtype/shape not supported */

/* ---- graph IR (nodes = ops, edges = dataflow) -------------------- */
enum sf_dtype { SF_F32 = 0, SF_I32 = 1 };

/* Kinds: PARAM/SLOT/SCALAR_STATE are persistent across iterations;
 * DATASET is read-only and replicated on every candidate device (never migrated);
 * INPUT/LABEL are fed each iteration (FEED op or request copy); ACT/GRAD are
 * intermediates; OUTPUT is fetched at iteration end (live until then). */
enum sf_tensor_kind {
  SF_PARAM = 0, SF_SLOT = 1, SF_SCALAR_STATE = 2, SF_DATASET = 3, SF_INPUT = 4,
  SF_LABEL = 5, SF_ACT = 6, SF_GRAD = 7, SF_OUTPUT = 8
};

/* The fixed op set of BASELINE.json north_star (+ GELU).  Operand
 * conventions:
 *  GEMM         in[A,B] out[C]        C = op(A) op(B) (+C if SF_GEMM_ACC); op = transpose
 *                                     if SF_GEMM_TA / SF_GEMM_TB; fp32-accurate (3xTF32)
 *  BIAS_ACT     in[z,b1(,b2,b3)] out[h(,u)]  u = z + b1 + b2 + b3; h = act(u): ReLU if
 *                                     SF_ACT_RELU, GELU (exact erf form) if SF_ACT_GELU, else
 *                                     identity; out[1] = u (GELU only: the backward needs it)
 *  BIAS_ACT_BWD in[dh,h] out[dz,db]   ReLU: dz = dh * [h > 0];
 *               in[dh,u] (SF_ACT_GELU) GELU: dz = dh * (Phi(u) + u phi(u));
 *                                     db = column sum of dz
 *  COLSUM       in[x] out[s]          s = column sum of x (s is [1, cols])
 *  SOFTMAX_CE   in[logits,labels] out[loss,dlogits]  mean sparse CE; (softmax-onehot)/B
 *  SOFTMAX      in[logits] out[probs]
 *  SGD_MOM      in[g] out[w,a]        a = mu * a + g; w = w - lr * a    (f = lr, mu)
 *  ADAM         in[g,step] out[w,m,v] TF Adam, t = step + 1 (f = lr, beta1, beta2, eps)
 *  FEED         in[pool,step] out[x]  x = pool rows [(step mod P) * rows, +rows)
 *  STEP_INC     out[step]             step += 1
 * Reductions are deterministic (fixed order): repeated runs are bitwise identical. */
enum sf_op_type {
  SF_OP_GEMM = 1, SF_OP_BIAS_ACT = 2, SF_OP_BIAS_ACT_BWD = 3, SF_OP_COLSUM = 4,
  SF_OP_SOFTMAX_CE = 5, SF_OP_SOFTMAX = 6, SF_OP_SGD_MOM = 7, SF_OP_ADAM = 8,
  SF_OP_FEED = 9, SF_OP_STEP_INC = 10
};
#define SF_GEMM_TA 1
#define SF_GEMM_TB 2
#define SF_GEMM_ACC 4
#define SF_ACT_RELU 1
#define SF_ACT_GELU 2 /* gelu(u) = u Phi(u) = 0.5 u (1 + erf(u / sqrt 2)) (BERT's activation) */

typedef struct sf_tensor_desc {
  int32_t rows, cols; /* 2-D row-major */
  int32_t dtype;      /* sf_dtype */
  int32_t kind;       /* sf_tensor_kind */
} sf_tensor_desc;

typedef struct sf_op_desc {
  int32_t type;    /* sf_op_type */
  int32_t n_in;    /* number of valid entries in in[] */
  int32_t in[6];   /* tensor ids (index into sf_graph_desc.tensors) */
  int32_t n_out;
  int32_t out[3];
  int32_t flags;   /* SF_GEMM_* / SF_ACT_RELU */
  int32_t phase;   /* layer-phase id: PER_LAYER_PHASE cuts where it changes */
  float f[4];      /* op scalars (lr, mu / lr, beta1, beta2, eps) */
} sf_op_desc;

typedef struct sf_graph_desc {
  const char* name;               /* copied; may be NULL */
  uint32_t n_tensors;
  const sf_tensor_desc* tensors;  /* host pointer, copied before return */
  uint32_t n_ops;
  const sf_op_desc* ops;          /* host pointer, topological order, copied */
} sf_graph_desc;

/* ---- runtime --------------------------------------------------------------------- */
typedef struct sf_runtime sf_runtime; /* opaque, one per process */
typedef uint32_t sf_graph_id;
typedef uint32_t sf_job_id;
typedef uint64_t sf_req_id;
#define SF_TARGET_HOST (-1) /* migrate the live set to pinned host memory (host tier) */

/* Host-tier transfer strategy. */
#define SF_HOST_CE 0 /* pack into device staging, copy-engine D2H; H2D, unpack */
#define SF_HOST_ZC 1 /* zero-copy: pack kernel stores straight into mapped pinned memory,
                        unpack kernel reads it back over PCIe */

/* Migration engine. */
#define SF_MIG_SM 0 /* descriptor-walk kernels: pack / unpack / fused peer store (default) */
#define SF_MIG_CE 1 /* copy engines only, zero SM work: cudaMemcpyAsync per segment in ~2 MB
                       groups (large tensors split), arena -> pinned staging payloads (the CPU writes header and
                       zero padding: same staging bytes as a pack), staging -> arena, or
                       arena -> peer arena; host_mode is ignored */

typedef struct sf_config {
  int32_t n_devices;             /* logical device slots */
  const int32_t* cuda_ordinals;  /* host array [n_devices]: CUDA device of each slot, or -1
                                    for a REMOTE slot: another process's device whose arena
                                    is mapped with sf_import_arena (process-per-GPU peers) */
  int32_t exclusive_gpu;         /* 1 (default behaviour): no two models' subgraphs co-run
                                    on a device; 0: free co-run baseline
                                    (multi-threaded TF) */
  int32_t auto_preempt;          /* 1: sf_submit_inference preempts the training job that
                                    owns the device */
  int32_t iteration_granularity; /* 1: preempt only at iteration boundaries (session time
                                    slicing baseline); 0: subgraph */
  int32_t host_mode;             /* SF_HOST_CE or SF_HOST_ZC */
  int32_t poison_released;       /* 1: fill released source arenas with 0xFF (tests) */
  int32_t trace_capacity;        /* events kept; 0 -> 1<<16 */
  int32_t max_inflight;          /* subgraphs queued on the device ahead of the host (1..4;
                                    0 -> 1): >1 removes the host gap between subgraphs; a
                                    preemption then waits for at most this many subgraphs */
  int32_t defer_migration;       /* 1: start the migration copy only after the device's
                                    queued inference drained (the paper defers the transfer
                                    past the preemption); 0: concurrent */
  uint64_t device_budget_bytes;  /* per device; 0 = unlimited */
  int32_t dispatch_spin_us;      /* an idle dispatcher busy-polls its request queue for this
                                    long before blocking on the runtime's condition variable
                                    (a futex wake-up adds tens of us to every request);
                                    0 = block at once, -1 = poll forever (one core per slot) */
  int32_t inflight_budget_us;    /* > 0: queue a subgraph behind in-flight ones only while
                                    their estimated device time (EMA of observed subgraph
                                    durations) stays within this budget, bounding what a
                                    preemption drains; 0 = window limit only */
  int32_t migrate_home;          /* 1: a job moved to a peer slot by a higher-priority job or
                                    an inference request migrates back to the slot it started
                                    on at its first boundary after that slot is free again (no
                                    queued inference, no present job of priority >= its own);
                                    0 (paper): it stays on the target */
  int32_t migration_engine;      /* SF_MIG_SM (default) or SF_MIG_CE */
  int32_t host_stage_inline;     /* 1: a job's host input stage runs on its driver thread while
                                    the job holds the device (with iteration_granularity = 1:
                                    session-based time slicing, the Gandiva-like baseline of
                                    PAPER.md:1385-1392); 0: feeds prefetch on their own thread
                                    (CPU executors scheduled freely) */
  int32_t host_duplex;           /* 1: a host-tier park that nothing waits for (the device's
                                    inference queue drained, no higher-priority job present,
                                    not an explicit sf_preempt) runs its round trip full
                                    duplex: each 2 MB chunk of the packed staging comes back
                                    H2D as soon as its D2H landed, so both PCIe directions run
                                    at once (max(S/d2h, S/h2d) instead of the sum); 0: D2H,
                                    then H2D */
  uint64_t infer_l2_persist_bytes; /* > 0: reserve this much of each device's L2 (clamped to
                                    cudaDevAttrMaxPersistingL2CacheSize) as a persisting
                                    set-aside for the inference graphs' weights: their request
                                    kernels carry an access-policy window over the arena and
                                    tag weight TMA loads evict_last, so the collocated training
                                    job's streaming traffic cannot evict them (Q29);
                                    0 = off */
  int32_t early_launch;          /* 1: a request that preempts the job owning the device is
                                    enqueued as soon as the job's driver can dispatch nothing
                                    more, behind a stream-ordered wait on the job's newest
                                    in-flight subgraph: the host launches overlap the drain
                                    and the chain starts on the GPU the moment the dispatched
                                    kernels finish; trace events of such
                                    requests carry the job in `iter` (invariant 1 through the
                                    device dependency); ignored with iteration_granularity;
                                    0: launch after the drain was observed on the host */
  int32_t drain_gate;            /* 1 (with early_launch and max_inflight >= 2): a training
                                    subgraph queued behind an in-flight one is enqueued behind a
                                    stream wait on a host gate word; a request that preempts the
                                    job holds that gate, so the GPU runs the request right after
                                    the RUNNING subgraph and the queued one after the request
                                    (it was dispatched before the arrival and still runs before
                                    the cut): the preemption latency is the
                                    running subgraph's residual only.  Dekker-style handshake
                                    over PCIe (reading Q38); when the GPU may already
                                    have passed the gate the request waits for both, as without
                                    the gate.  0: off */
} sf_config;

/* Create a runtime: enables peer access between distinct CUDA devices of the slots,
 * creates per-slot streams (training, high-priority inference, migration) and one
 * dispatcher thread per slot.  *out owned by the caller, freed by sf_destroy. */
sf_status sf_create(const sf_config* cfg, sf_runtime** out);
/* Wait for all jobs and requests, join threads, free runtime-owned memory. */
void sf_destroy(sf_runtime* rt);
/* Thread-local text of the last error (valid until the next failing call). */
const char* sf_last_error(void);
int32_t sf_abi_version(void);

/* Validate and copy a graph (shapes, dtypes, op arity, read-before-write).
 * priority: larger = more important.  Inference requests always rank
 * above every training job (reading Q13).  Between training jobs (PAPER.md:1184-1222,
 * Fig. 7 scenario): a job of a higher-priority graph started on a slot is "allowed to start
 * immediately after submission" — every lower-priority job on that slot
 * stops at its next subgraph boundary and migrates to its auto_target (peer slot: resumes
 * there at once; SF_TARGET_HOST: parked, swapped back in once no higher-priority job is
 * present on the slot), or, when its auto_target is the slot itself, waits in place.
 * SF_EUNSUPPORTED for ops outside the fixed set; SF_EINVAL for malformed graphs. */
sf_status sf_register_graph(sf_runtime* rt, const sf_graph_desc* g, int32_t priority,
                            sf_graph_id* out);

#define SF_PART_PER_LAYER_PHASE 0
#define SF_PART_MAX_OPS 1
typedef struct sf_partition_opts {
  int32_t policy;        /* SF_PART_PER_LAYER_PHASE (maximal runs of equal phase) or
                            SF_PART_MAX_OPS (split runs to <= max_ops ops; optimizer runs whole) */
  int32_t max_ops;
  int32_t update_chunks; /* > 1: split each optimizer run into this many byte-balanced
                            subgraphs: op j (weight = nbytes of its variable, 0 for STEP_INC,
                            C_j = weight of the run's earlier ops, W = run total) goes to chunk
                            min(U-1, floor(U*C_j/W)); bounds the longest subgraph, i.e. the
                            preemption latency */
} sf_partition_opts;
typedef struct sf_partition_info {
  int32_t n_subgraphs;
  uint64_t arena_bytes;      /* device bytes each bound device must provide */
  uint64_t staging_bytes;    /* bytes of the largest staging buffer (max over cuts) */
  uint64_t persistent_bytes; /* PARAM + SLOT + SCALAR_STATE */
  uint64_t max_live_bytes;   /* max over cuts of sum(nbytes of L_k) */
} sf_partition_info;

/* Partition into subgraphs S_0..S_{n-1}, compute the live set L_k of every cut and the
 * arena layout.  May be called once per graph. */
sf_status sf_partition(sf_runtime* rt, sf_graph_id g, const sf_partition_opts* o,
                       sf_partition_info* out);
/* Op range [begin, end) of subgraph k. */
sf_status sf_subgraph_range(sf_runtime* rt, sf_graph_id g, int32_t k, int32_t* op_begin,
                            int32_t* op_end);
/* L_k as ascending tensor ids (host array ids[cap]); *n = |L_k|, *bytes = sum nbytes. */
sf_status sf_live_set(sf_runtime* rt, sf_graph_id g, int32_t k, uint32_t* ids, uint32_t cap,
                      uint32_t* n, uint64_t* bytes);
/* Byte offset of a tensor inside every arena of this graph. */
sf_status sf_tensor_offset(sf_runtime* rt, sf_graph_id g, uint32_t tensor_id, uint64_t* off);
/* Staging layout of cut k: total bytes and payload offset of the e-th live tensor. */
sf_status sf_staging_layout(sf_runtime* rt, sf_graph_id g, int32_t k, uint64_t* total,
                            uint64_t* payload_offsets, uint32_t cap);

/* Bind memory of device slot `dev` to graph g and build its versions: one CUDA graph per
 * subgraph (the per-device executor replica) plus the pack / unpack /
 * peer-store descriptor lists of every cut.
 *   arena        device pointer, >= arena_bytes, 256-B aligned (caller fills DATASET /
 *                PARAM / SLOT / SCALAR_STATE contents at sf_tensor_offset() offsets)
 *   staging      device pointer, >= staging_bytes, or NULL (then host tier uses ZC)
 *   host_staging pinned host pointer, >= staging_bytes, or NULL (no host tier)
 * Peer-store lists to a slot are built when both slots are bound.  Returns SF_ENOMEM when
 * the persistent bytes of all graphs bound to the slot exceed device_budget_bytes. */
sf_status sf_bind(sf_runtime* rt, sf_graph_id g, int32_t dev, void* arena, void* staging,
                  void* host_staging);

/* ---- training jobs, preemption --------------------------------------------------- */
enum sf_job_state {
  SF_JOB_RUNNING = 0, SF_JOB_STOPPING = 1, SF_JOB_MIGRATING = 2, SF_JOB_PREEMPTED = 3,
  SF_JOB_DONE = 4, SF_JOB_FAILED = 5,
  SF_JOB_MIGRATED_OUT = 6 /* state copied into a REMOTE slot; the partner adopts the job */
};
typedef struct sf_job_info {
  int32_t state;        /* sf_job_state */
  int32_t dev;          /* current device slot (source while migrating) */
  int64_t iter;         /* next (iter, k) to run */
  int32_t k;
  int32_t n_preemptions;
  uint64_t migrated_bytes;      /* cumulative live bytes moved */
  double last_pack_us;          /* CUDA-event durations of the last migration's kernels */
  double last_xfer_us;
  double last_unpack_us;
  uint64_t last_stop_ns;        /* CLOCK_MONOTONIC: cut decided (in-flight S_k done) */
  uint64_t last_resume_ns;      /* CLOCK_MONOTONIC: first resumed subgraph began on the device
                                   (host-observed completion of a marker recorded right before it,
                                   i.e. after the stream-ordered copy / unpack finished) */
  int64_t n_reparks;            /* host-tier preemptions that found the parked copy of the
                                   same cut still current (nothing ran since the swap-in) and
                                   re-parked without pack / D2H */
  uint64_t submit_ns;           /* CLOCK_MONOTONIC at sf_start_training / sf_adopt_job */
  int32_t priority;             /* the graph's registered priority */
  int32_t home;                 /* slot the job started on */
} sf_job_info;

typedef struct sf_cut_info {
  int64_t iter;          /* the cut sits before S_k of this iteration */
  int32_t k;
  int32_t n_tensors;     /* |L_k| */
  uint64_t live_bytes;   /* sum nbytes(L_k) */
  uint64_t t_req_ns;     /* CLOCK_MONOTONIC when the preemption was requested */
  uint64_t t_stop_ns;    /* when the job stopped at the boundary */
  int32_t src_dev, dst_dev;
} sf_cut_info;

/* A preemption scheduled at a fixed cut: before S_k of iteration `iter`, migrate the live
 * set to `target` (peer slot or SF_TARGET_HOST) and resume right away (peer: on the
 * target; host: swap back into the same slot once its inference queue drained). */
typedef struct sf_cut_request {
  int64_t iter;
  int32_t k;
  int32_t target;
} sf_cut_request;

/* Start a training job of graph g on bound slot `dev` for `iters` iterations (job
 * driver thread).  `auto_target` = where an auto-preemption migrates it (peer slot or
 * SF_TARGET_HOST).  `sched` (host array, n_sched entries, ascending (iter, k), copied)
 * lists deterministic preemptions, e.g. for "preempted N times == unpreempted" checks. */
sf_status sf_start_training(sf_runtime* rt, sf_graph_id g, int32_t dev, int64_t iters,
                            int32_t auto_target, const sf_cut_request* sched, int32_t n_sched,
                            sf_job_id* out);
/* Preempt: block until the job stops at its next subgraph boundary (kernels of the
 * in-flight subgraph finish) and its migration to `target` (peer slot
 * or SF_TARGET_HOST) is enqueued; does not wait for the migration.  The job then stays
 * SF_JOB_PREEMPTED until sf_resume.  SF_ESTATE if not RUNNING; SF_EINVAL if target is the
 * current slot or unbound; SF_EBUSY if a migration is in flight. */
sf_status sf_preempt(sf_runtime* rt, sf_job_id job, int32_t target, sf_cut_info* out);
/* Resume a preempted job on `dev` (peer tier: the migration target; host tier: any bound
 * slot) — stream-ordered after the migration, no host sync on the copy: "the new session is
 * populated with the tasks of the aborted session run so that no work is lost" and later
 * sessions run on the new device (section 3.3).  SF_ESTATE if the
 * job is not preempted. */
sf_status sf_resume(sf_runtime* rt, sf_job_id job, int32_t dev);
sf_status sf_job_query(sf_runtime* rt, sf_job_id job, sf_job_info* out);
/* Copy tensor `tensor_id` of a job's graph (n bytes, n == its byte size) from the arena of the
 * slot the job occupies into host memory host_dst (blocking).  The copy is ordered after every
 * subgraph the job has dispatched (a snapshot at a subgraph boundary when the job runs; the
 * final value once it is done) — the paper's users fetch results through the session
 * (Listing 1).  SF_EBUSY while the job's state is parked in host memory or
 * moving (host tier, migration in flight); SF_EINVAL for a bad id or size. */
sf_status sf_read_tensor(sf_runtime* rt, sf_job_id job, uint32_t tensor_id, void* host_dst, size_t n);
/* Wait until the job finished all iterations (SF_ETIMEOUT after timeout_ns; <0 = inf). */
sf_status sf_wait_job(sf_runtime* rt, sf_job_id job, int64_t timeout_ns);
/* Ask a running job to stop at its next iteration boundary and finish. */
sf_status sf_stop_job(sf_runtime* rt, sf_job_id job);

/* ---- process-per-GPU peers (CUDA IPC) ------------------------------------------------
 * The paper migrates a job between devices of one machine; with
 * one process per GPU the target arena lives in another process.  Each process exports its
 * arena once; the partner maps it into a REMOTE slot; a preemption to that slot runs the
 * peer-store kernel straight into the partner's HBM over NVLink, waits for the copy, and
 * leaves the job SF_JOB_MIGRATED_OUT with its cut in sf_cut_info; the partner process then
 * calls sf_adopt_job with that cut (handoff message carried by the caller, e.g.
 * torch.distributed). */
typedef struct sf_ipc_arena {
  uint8_t handle[64];     /* cudaIpcMemHandle_t of the allocation holding the arena */
  uint64_t offset;        /* arena offset inside that allocation */
  uint64_t arena_bytes;
  int32_t cuda_ordinal;   /* device of the exporting process (informational) */
  int32_t pad;
} sf_ipc_arena;
/* Export the arena of graph g bound on local slot dev. */
sf_status sf_export_arena(sf_runtime* rt, sf_graph_id g, int32_t dev, sf_ipc_arena* out);
/* Map a partner's exported arena as REMOTE slot `slot` of graph g (opened on the device of
 * the first local slot g is bound to) and build peer-store lists from every local binding. */
sf_status sf_import_arena(sf_runtime* rt, sf_graph_id g, int32_t slot, const sf_ipc_arena* a);
/* Start a job whose live state at cut (iter, k) is already in dev's arena (copied there by a
 * partner's peer store); runs until `iters` iterations are complete. */
sf_status sf_adopt_job(sf_runtime* rt, sf_graph_id g, int32_t dev, int64_t iters, int64_t iter,
                       int32_t k, int32_t auto_target, sf_job_id* out);

/* ---- host input stages: interleaving and input reuse ------
 * The paper's CPU executor (data loading + preprocessing) of a job: "executors
 * on different devices can be scheduled freely ... any CPU executor [may] run while a GPU is
 * occupied", overlapping one job's preprocessing with another job's GPU subgraphs.  A feed runs
 * a host stage callback that writes iteration `iter`'s fed tensors (INPUT / LABEL tensors no op
 * writes) into pinned buffers, prefetching up to `depth` iterations on a runtime thread that
 * never holds a device.  At S_0 of each iteration the job copies them into its arena on its
 * training stream (they then migrate like any in-flight tensor).
 * Shared feed (input reuse, Fig. 5): one host stage feeds several graphs;
 * each batch is copied once into an immutable device buffer ("an immutable copy of the tensor in
 * GPU global memory ... public to all GPU executors sharing the tensor") and the members run
 * their iterations in lockstep round-robin (member 0's iteration i, member 1's iteration i,
 * ..., then batch i+1).  Members are the graphs attached to the feed, in attach order; they
 * must run the same number of iterations and start at iteration 0. */
typedef uint32_t sf_feed_id;
/* Host stage: fill dst[i] (pinned host, bytes[i] bytes) for iteration `iter`; return 0 on
 * success (non-zero fails the job).  Called from one runtime thread at a time per feed. */
typedef int32_t (*sf_host_stage_fn)(void* user, int64_t iter, void* const* dst,
                                    const uint64_t* bytes, int32_t n);
typedef struct sf_feed_desc {
  sf_host_stage_fn fn;
  void* user;              /* passed to fn; caller-owned, valid until sf_destroy */
  int32_t n;               /* fed tensors per iteration, 1..8 */
  const uint64_t* bytes;   /* host [n], copied */
  int32_t depth;           /* prefetch ring slots 1..8 (0 -> 2) */
  int32_t shared;          /* 1: input-reuse group (immutable device copy, lockstep members) */
  int32_t dev;             /* shared: slot whose device holds the immutable copy */
  int32_t pad;
} sf_feed_desc;
sf_status sf_create_feed(sf_runtime* rt, const sf_feed_desc* d, sf_feed_id* out);
/* Feed graph g's tensors tensor_ids[0..n) (host array; INPUT / LABEL tensors no op writes, byte
 * sizes equal to the feed's) from feed f.  Before sf_start_training; a non-shared feed takes one
 * graph.  SF_EINVAL on size / kind mismatch. */
sf_status sf_attach_feed(sf_runtime* rt, sf_graph_id g, sf_feed_id f, const uint32_t* tensor_ids);

/* Built-in host stage (synthetic image pipeline, reading Q27): batch b = iter mod P of
 * a u8 image pool [P * batch][cols] is decoded to fp32 x = u8 / 255 with a seeded horizontal
 * flip per sample (row r of the pool flips when the low bit of the (r+1)-th splitmix64 output of
 * `seed` is set; images are img_w pixels wide), labels copied; dst = {x [batch][cols] f32,
 * y [batch][1] i32}.  user = const sf_u8_stage*. */
typedef struct sf_u8_stage {
  const uint8_t* images;   /* host [pool_rows][cols] */
  const int32_t* labels;   /* host [pool_rows] */
  int64_t pool_rows;       /* multiple of batch */
  int32_t batch, cols, img_w;
  uint32_t seed;
} sf_u8_stage;
int32_t sf_stage_u8_normalize(void* user, int64_t iter, void* const* dst, const uint64_t* bytes,
                              int32_t n);

/* ---- inference (the preempter) --------------------------------------------------- */
typedef struct sf_timing {
  uint64_t arrival_ns;   /* scheduled arrival (CLOCK_MONOTONIC) */
  uint64_t start_ns;     /* the request chain's start on the device (GPU timeline mapped to
                            CLOCK_MONOTONIC, Q37; host dispatch time if unmapped) */
  uint64_t end_ns;       /* completion observed */
  int32_t dev;
  int32_t preempted_job; /* job cut by this request, or -1 */
  int64_t cut_iter;
  int32_t cut_k;
  float device_us;       /* device time of the request's kernel chain (input copy .. output
                            copy), CUDA events on the inference stream */
  float launch_us;       /* host time the dispatcher took to issue the chain (first event
                            record .. last launch returned) */
  float dispatch_us;     /* host time from the dispatch decision to the first enqueue */
} sf_timing;

/* Enqueue a batch-1 request of inference graph g on slot dev (non-blocking).  The request is
 * the high-priority job that "is allowed to start immediately after submission" while the
 * preempted one is suspended at its next boundary (section 3.4; arrival
 * triggers preemption, section 3.3).
 * in: pointer (device or pinned host) to the INPUT tensor's bytes; out: pointer (device
 * or pinned host) receiving the OUTPUT tensor's bytes; both caller-owned until sf_wait.
 * arrival_ns = scheduled arrival time (CLOCK_MONOTONIC ns; 0 = now).  With
 * auto_preempt the training job owning dev is preempted to its auto_target. */
sf_status sf_submit_inference(sf_runtime* rt, sf_graph_id g, int32_t dev, const void* in,
                              void* out, uint64_t arrival_ns, sf_req_id* req);
/* Wait for a request; fills *timing. */
sf_status sf_wait(sf_runtime* rt, sf_req_id req, int64_t timeout_ns, sf_timing* timing);

/* ---- trace (schedule invariants; oracle/schedule.py checks it) ------------------- */
enum sf_event_kind { SF_EV_TRAIN = 0, SF_EV_INFER = 1, SF_EV_MIGRATE = 2,
                     SF_EV_HOST = 3 /* host stage of a feed: dev = -1 - feed id (prefetch
                                       thread) or the job's slot (inline), k = -1 */ };
typedef struct sf_trace_event {
  int32_t dev, job, kind, k;   /* job: training job id, or 1<<20 | request for inference */
  int64_t iter;
  uint64_t t0_ns, t1_ns;       /* host CLOCK_MONOTONIC: launch .. completion observed */
  uint64_t arrival_ns;         /* inference: scheduled arrival; train: host dispatch time
                                  (<= t0 when queued behind an in-flight predecessor) */
  /* inference: iter = -1, or the training job whose subgraphs dispatched before t0 this
     request was ordered after on the device (early_launch); t0 is then its dispatch time;
     k = 1 when the drain gate held the job's queued subgraphs behind this request */
  uint64_t d0_ns, d1_ns;       /* DEVICE execution interval on the CLOCK_MONOTONIC axis: timing
                                  events recorded on the stream right before the subgraph's
                                  graph (request chain) and right after it, mapped through a
                                  %globaltimer anchor (reading Q37); a superset of
                                  the kernels' execution; 0 = unavailable (train / infer only) */
} sf_trace_event;
sf_status sf_get_trace(sf_runtime* rt, sf_trace_event* buf, size_t cap, size_t* n_out);
uint64_t sf_now_ns(void); /* CLOCK_MONOTONIC */

/* ---- kernel entry points (operate on plain device pointers; async on `stream`) ---- */
/* Multi-tensor copy descriptor: copy nbytes (multiple of 4) from src to dst, and write
 * zeros from nbytes up to span (span >= nbytes, multiple of 16); src/dst 16-B aligned.
 * This single descriptor walk is the pack (arena -> staging, span = round_up(nbytes,256)),
 * unpack (staging -> arena) and peer-store (arena -> peer arena over NVLink) kernel. */
typedef struct sf_copy_desc {
  const void* src;
  void* dst;
  uint64_t nbytes;
  uint64_t span;
} sf_copy_desc;
/* descs: HOST array [n].  patch_iter >= 0: overwrite bytes [16, 24) of descriptor 0's
 * destination with patch_iter (the staging header's iter field). */
sf_status sf_op_mtcopy(const sf_copy_desc* descs, int32_t n, int64_t patch_iter, void* stream);
/* C = op(A) op(B) (+C); lda/ldb/ldc = row strides (elements) of the stored matrices.
 * Split-K shapes use a runtime-owned workspace cached per (device, stream) and grown on
 * demand (never freed before process exit); calls on one stream share it in stream order. */
sf_status sf_op_gemm(const float* A, const float* B, float* C, int32_t M, int32_t N,
                     int32_t K, int32_t lda, int32_t ldb, int32_t ldc, int32_t flags,
                     void* stream);
/* C = act(op(A) op(B) (+C) + b1 (+ b2) (+ b3)), act = ReLU if relu else identity; the GEMM
 * of a forward layer with its BIAS_ACT epilogue (PAPER.md:1213-1220 workload; SURVEY.md 8(a)
 * K5).  b1 is required (SF_EINVAL otherwise); biases are 1 x N rows.  Batch <= 8 fuses the
 * epilogue into the GEMV's cluster reduction; otherwise it runs as a second elementwise
 * kernel in place (requires ldc == N). */
sf_status sf_op_gemm_bias_act(const float* A, const float* B, float* C, int32_t M, int32_t N,
                              int32_t K, int32_t lda, int32_t ldb, int32_t ldc, int32_t flags,
                              const float* b1, const float* b2, const float* b3, int32_t relu,
                              void* stream);
/* Fused batch-M inference chain (M <= 8): h[l] = act_l(h[l-1] W[l] + b[l]) for l = 0..n-1
 * with h[-1] = x, act_l = ReLU if relu[l] else identity, then probs = softmax(h[n-1]) row-wise
 * when probs != NULL — the preempter's forward pass of SURVEY.md 8(a) a6
 * in one persistent kernel.  widths: host [n+1] (K_0, N_0 = K_1, ..., N_{n-1}); W[l]:
 * device K_l x N_l row-major (N_l % 4 == 0, 16-B aligned); b[l]: device 1 x N_l or NULL (b
 * itself may be NULL); relu: host [n] or NULL; h[l]: device M x N_l, all written.  n <= 6,
 * otherwise SF_EUNSUPPORTED. */
/* Diagnostics: while dev_buf != NULL every fused-chain launch writes per-CTA phase
 * timestamps (%globaltimer ns) to dev_buf, uint64 [n_SMs][64] = [cta][layer * 8 + event]
 * (events: 0 layer start, 1 inputs ready, 2 x staged, 3 first W box, 4 units done,
 * 5 partial published, 6 column block reduced, 7 chain done).  NULL turns it off. */
sf_status sf_debug_chain_trace(void* dev_buf);
sf_status sf_op_mlp_chain(const float* x, int32_t M, int32_t n_layers, const int32_t* widths,
                          const float* const* W, const float* const* b, const int32_t* relu,
                          float* const* h, float* probs, void* stream);
/* act: 0 identity, SF_ACT_RELU, SF_ACT_GELU. */
sf_status sf_op_bias_act(const float* z, const float* b1, const float* b2, const float* b3,
                         float* h, int32_t rows, int32_t cols, int32_t act, void* stream);
sf_status sf_op_bias_act_bwd(const float* dh, const float* h, float* dz, float* db,
                             int32_t rows, int32_t cols, void* stream);
/* GELU backward fused with the bias gradient: dz = dh * gelu'(u); db = column sum of dz. */
sf_status sf_op_gelu_bwd(const float* dh, const float* u, float* dz, float* db, int32_t rows,
                         int32_t cols, void* stream);
sf_status sf_op_colsum(const float* x, float* s, int32_t rows, int32_t cols, void* stream);
sf_status sf_op_softmax_ce(const float* logits, const int32_t* labels, float* loss,
                           float* dlogits, int32_t rows, int32_t cols, void* stream);
sf_status sf_op_softmax(const float* logits, float* probs, int32_t rows, int32_t cols,
                        void* stream);
sf_status sf_op_sgd_mom(float* w, float* a, const float* g, int64_t n, float lr, float mu,
                        void* stream);
sf_status sf_op_adam(float* w, float* m, float* v, const float* g, const int32_t* step,
                     int64_t n, float lr, float beta1, float beta2, float eps, void* stream);
/* Fill n bytes at dst (device) with byte value (0xFF = poison). */
sf_status sf_op_fill(void* dst, uint64_t n, int32_t value, void* stream);
/* Batch <= 8 GEMMs with constant weights (inference layers) stream a blocked copy of the
 * weights (contiguous per-CTA blocks for the LDG GEMV, reading Q39), allocated by
 * sf_bind and laid out from the arena by this call (or, failing that, at the binding's first
 * request).  Call it after writing or rewriting the weights in the arena of slot dev; it blocks
 * until the copy is done. */
sf_status sf_refresh_constants(sf_runtime* rt, sf_graph_id g, int32_t dev);
/* Diagnostics: a device slot's scheduler state (owner token: a training job id, 1 << 20 while
 * inference runs, -1 free; requests queued; drain-gate words). */
typedef struct sf_slot_info {
  int32_t owner, queued, gate_held, pad;
  uint32_t gate_value, gate_arrived, next_ticket;
  uint32_t gate_valve; /* holds the dispatcher released after a chain waited 5 ms behind its own
                          hold (streams sharing a hardware queue with the held training stream) */
} sf_slot_info;
sf_status sf_slot_query(sf_runtime* rt, int32_t slot, sf_slot_info* out);
/* Diagnostics: the kernel path of the last GEMM the CALLING THREAD launched (sf_op_gemm,
 * sf_op_gemm_bias_act, or a subgraph op launched directly on this thread).
 * kind: 1 tcgen05 TMA tile GEMM (bn = tile width 64 / 128 / 256, splits = split-K factor),
 *       2 tcgen05 GEMM with LDG producers (pitches TMA cannot map), 3 TMA cluster GEMV,
 *       4 row-contiguous GEMV (TB), 5 register cluster GEMV, 6 split-K GEMV + reduce,
 *       7 plain GEMV, 8 LDG GEMV over blocked constant weights; 0 = none yet.
 * a_mn / b_mn: operand stored MN-major (A as [K][M], i.e. TA; B as [K][N], i.e. not TB). */
typedef struct sf_gemm_path {
  int32_t kind, bn, splits, a_mn, b_mn, pad;
} sf_gemm_path;
sf_status sf_last_gemm_path(sf_gemm_path* out);
/* Diagnostics (migration roofline): run the bound pack list (arena ->
 * device staging, header + payloads + zero padding) and unpack list (staging -> arena) of cut k
 * on slot dev once each, on the slot's migration stream, and return their kernel-only durations
 * (in-kernel %globaltimer).  l2 = 0: as is (warm: a walk right after another); 1: cold, clean L2
 * (read a buffer of twice the L2 size before each walk); 2: cold, dirty L2 (write it: the
 * write-back shares HBM with the walk, as after a training subgraph).  The unpack restores the
 * bytes the pack read, so the arena is unchanged.  Blocks until done.  SF_EBUSY if a job of the
 * graph is running; SF_EINVAL if dev has no device staging. */
typedef struct sf_migration_probe {
  double pack_us, unpack_us;
  uint64_t live_bytes;     /* sum nbytes(L_k) */
  uint64_t staging_bytes;  /* bytes the pack writes (header + payloads + padding) */
} sf_migration_probe;
sf_status sf_probe_migration(sf_runtime* rt, sf_graph_id g, int32_t dev, int32_t k, int32_t l2,
                             sf_migration_probe* out);
/* Diagnostics (C5 migration sweep): move the live set of cut k from local slot
 * src into slot dst's arena (a local slot of another device, or a REMOTE slot mapped with
 * sf_import_arena) once, on src's migration stream, and return the duration.  engine:
 *   0 the peer-store descriptor walk (the product path; kernel-only %globaltimer time),
 *   1 copy engines, cudaMemcpyAsync per segment in ~2 MB groups (large tensors split),
 *   2 copy engines, one cudaMemcpyAsync per tensor (per-tensor cudaMemcpyPeerAsync),
 *   3 copy engines, ONE cudaMemcpyAsync of the arena span the live tensors cover;
 * CE times are CUDA events around the copies.  Blocks until done.  *bytes_moved = live bytes
 * (engine 3: the span).  SF_EBUSY if a job of the graph is running. */
sf_status sf_probe_peer(sf_runtime* rt, sf_graph_id g, int32_t src, int32_t dst, int32_t k,
                        int32_t engine, double* us, uint64_t* bytes_moved);
/* Number of kernels this process launched through the library so far. */
uint64_t sf_kernel_launches(void);

#ifdef __cplusplus
}
#endif
#endif /* SF_H_ */
