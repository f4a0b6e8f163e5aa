/*
 * duet.h — C ABI of libduet.so, the B200-native DUET hot path.
 *
 * DUET (IPDPS'21, /root/reference/PAPER.md) runs a multi-branch DNN inference graph
 * concurrently: the input is a pre-compiled DNN model (§IV); a coarse-grained
 * partitioner cuts it into phases of subgraphs (§IV-A); a compiler-aware profiler
 * times every compiled subgraph on every device (§IV-B); the greedy-correction
 * scheduler maps subgraphs to devices (§IV-C, Algorithm 1 at PAPER.md:86); an
 * executor runs the schedule (§IV-D).  Here a "device" is a slot = (GPU, CUDA
 * stream) on a B200 (BASELINE.json:5 north_star), and the executor is one CUDA graph replay.
 *
 * General conventions
 *  - Every entry point returns duet_status (no C++ exception crosses the ABI).  On failure the
 *    out-parameter is set to NULL, no partial state is kept, and duet_last_error() explains.
 *  - Opaque handles are library-owned and freed by the matching *_destroy; destroy(NULL) is a
 *    no-op.  A handle must outlive every handle created from it (graph > partition > profile
 *    > schedule).
 *  - Weights, inputs, outputs and streams are CALLER-owned (allocated through torch in the
 *    Python binding) and must outlive the handles that reference them.  The library owns only
 *    CUDA events, CUDA graphs, TMA descriptors, and its intermediate / preprocessed-weight
 *    device buffers.
 *  - Tensors are dense row-major (C-contiguous).  data is a device pointer when device >= 0
 *    and a host pointer when device == DUET_HOST (host buffers should be pinned for async).
 *  - Shapes are static ("we freeze the model with a fixed batch size"): every
 *    shape including the batch is fixed by the IR; other shapes are rejected (DUET_ESHAPE).
 *  - Handles are not thread-safe.  One duet_run may be in flight per graph (intermediate
 *    buffers are per graph and reused by every run).
 *  - Determinism: duet_partition depends only on (IR, options); duet_schedule only on
 *    (partition, profile table, options).  Both equal the CPU oracle (oracle/) bit for bit.
 *
 * IR text (the analogue of the paper's Relay -> adjacency-list translation):
 *   line    := comment | param | node | output
 *   comment := '#' anything
 *   param   := 'param' '@'NAME ':' DTYPE '[' d0,d1,... ']'
 *   node    := '%'NAME '=' OP '(' ARG, ... ')' [ '{' key=value, ... '}' ] ':' DTYPE '[' dims ']'
 *   ARG     := '%'NAME (a node's output) | '@'NAME (a parameter)
 *   output  := 'output' '%'NAME, ...
 *   DTYPE   := f32 | bf16 | i32 | i64
 *   Names may be used before their definition; the graph must be acyclic (else DUET_ECYCLE).
 *   Operators (B = batch; semantics = the float64 oracle, oracle/forward.py):
 *     input()                                      graph input, bound per duet_run
 *     hash_mod(%raw i64[B,F]) {V}                  id = raw mod V (floor) -> i32[B,F]
 *     gather_sum(%ids, @T[F,R], @b f32[1])         y[b] = b0 + sum_f T[f,ids[b,f]] -> f32[B,1]
 *     gather_concat(%ids, @E[F,R,D])               X[b,fD+k] = E[f,ids[b,f],k] -> [B,F*D]
 *     embed_seq(%tok i32[B,S], @E[V,D])            X[t,b,:] = E[tok[b,t],:] -> [S,B,D]
 *     linear(%x[M,K], @W[N,K], @b f32[N]) {act}    act(x W^T + b) -> [M,N]
 *     mlp(%x, @W0,@b0, ..., @Wn,@bn) {act,last_act} chain of linear layers
 *     reduce_sum(%x[B,K], @b f32[1])               y[b] = b0 + sum_k x[b,k] -> f32[B,1]
 *     lstm(%x[S,B,E], @Wih[4H,E], @Whh[4H,H], @bih f32[4H], @bhh f32[4H])  h_S -> [B,H]
 *                                                  (PyTorch gate order i,f,g,o; h0=c0=0)
 *     gru(%x[S,B,E], @Wih[3H,E], @Whh[3H,H], @bih f32[3H], @bhh f32[3H])   h_S -> [B,H]
 *                                                  (PyTorch r,z,n; b_hn inside r*(.))
 *     lstm / gru {seq=1}                           every h_t -> [S,B,H] (a lower layer of a stacked
 *                                                  RNN, Fig. 14)
 *     lstm / gru {tile_n=64|128|256}               gate-tile width of the persistent recurrence
 *                                                  (an SM budget when branches share the GPU;
 *                                                  absent = automatic; other values DUET_EINVAL)
 *     conv2d_bn(%x[N,H,W,C], @W[Co,kh,kw,C], @gamma,@beta,@mean,@var f32[Co]) {stride,pad,act}
 *                                                  NHWC conv + inference BN (eps 1e-5) + act
 *     add(%a, %b) {act}   maxpool(%x) {k,stride,pad}   avgpool(%x[N,H,W,C]) -> [N,C]
 *     dot_join(%s[B,1], %a[B,K], @w f32[K], @b f32[1])   sigma(s + a.w + b)    -> f32[B,1]
 *     cosine_join(%a[B,K], %b[B,K])                      a.b/(|a||b|), 0 if 0  -> f32[B,1]
 *     concat_head(%a1, ..., @w f32[sum K], @b f32[1]) {act}  act(concat(a).w + b) -> f32[B,1]
 *     sum_join(%l1, ...)  sigma(sum l_i)    mean_join(%l1, ...)  sigma(mean l_i)  -> f32[B,1]
 *     sigmoid(%x)
 *   MT-DNN (Fig. 3; LayerNorm eps 1e-12):
 *     bert_embed(%tok i32[B,S], %seg i32[B,S], @Etok[V,H], @Epos[>=S,H], @Eseg[2,H], @g f32[H], @b f32[H])
 *                                                  LN(Etok[tok] + Epos[s] + Eseg[seg]) -> [B*S,H]
 *     attention(%qkv[B*S,3H]) {heads,seq}          softmax(Q K^T/sqrt(dh)) V per head -> [B*S,H]
 *                                                  (no mask; seq <= 512, dh in {32,64,128})
 *     add_layernorm(%a[M,H], %b[M,H], @g, @b)      LN(a + b) -> [M,H]
 *     select_rows(%x[M,K]) {stride,offset}         rows offset + i*stride -> [rows,K]
 *     opaque(%in...)   structure + declared output bytes only; no kernel (scheduler fixtures
 *                      used with duet_profile_from_table; duet_run rejects it)
 *   act := none | relu | sigmoid | tanh | gelu (erf form).  Activations are stored in the node's declared dtype
 *   (bf16 graphs: bf16 weights/activations, fp32 accumulation, fp32 LSTM cell state).
 */
#ifndef DUET_H_
#define DUET_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define DUET_ABI_VERSION 2
#define DUET_HOST (-1)
#define DUET_MAX_DIMS 8

typedef struct duet_graph_t duet_graph_t;
typedef struct duet_partition_t duet_partition_t;
typedef struct duet_profile_t duet_profile_t;
typedef struct duet_schedule_t duet_schedule_t;

typedef enum {
  DUET_OK = 0,
  DUET_EINVAL = -1,       /* bad argument (NULL handle, bad option value, ...)            */
  DUET_EPARSE = -2,       /* IR text does not follow the grammar above                      */
  DUET_ECYCLE = -3,       /* IR graph has a cycle                                           */
  DUET_ESHAPE = -4,       /* a tensor's shape differs from the IR declaration               */
  DUET_EDTYPE = -5,       /* a tensor's dtype differs from the IR declaration               */
  DUET_EUNBOUND = -6,     /* a parameter was not bound before profile / run                 */
  DUET_ECUDA = -7,        /* CUDA runtime error (message appended)                          */
  DUET_ENCCL = -8,        /* reserved: NCCL error                                           */
  DUET_ENOMEM = -9,       /* host or device allocation failed                               */
  DUET_EUNSUPPORTED = -10,/* valid request this build does not implement (reason given)     */
  DUET_ESTATE = -11       /* call sequence error (e.g. run before schedule)                 */
} duet_status;

typedef enum { DUET_F32 = 0, DUET_BF16 = 1, DUET_I32 = 2, DUET_I64 = 3 } duet_dtype;

/* Non-owning view of a dense row-major tensor. device = CUDA ordinal, or DUET_HOST. */
typedef struct {
  void* data;
  int device;
  duet_dtype dtype;
  int ndim;
  int64_t shape[DUET_MAX_DIMS];
} duet_tensor;

/* A placement target ("device" of Algorithm 1): a caller-owned, non-default
 * cudaStream_t on CUDA device `gpu`.  slots[0] is the HOME slot: graph inputs are resident
 * there and the final outputs must reach it. */
typedef struct {
  int gpu;
  void* stream;
} duet_slot;

/* Communication cost of one boundary tensor (Fig. 5: latency linear in size):
 * cost_ns = alpha_ns + ceil(bytes * ps_per_byte / 1000); 0 between subgraphs on one slot. */
typedef struct {
  int64_t alpha_ns;
  int64_t ps_per_byte;
} duet_link;
typedef struct {
  duet_link same_gpu;   /* another stream on the same GPU: an event wait, no bytes move */
  duet_link cross_gpu;  /* another GPU: NVLink copy of the boundary tensor             */
} duet_comm_model;

typedef struct {
  int granularity;   /* 0 = coarse, 1 = one subgraph per operator node    */
  int batch_shards;  /* 1 = off; k in [2, 64]: every multi-path subgraph becomes k row shards
                      * (duet_partition_shards).  A sharded
                      * partition is a scheduling model for multi-GPU placement: it schedules
                      * from duet_profile_from_table; duet_profile / duet_schedule_measured /
                      * duet_run reject it with DUET_EUNSUPPORTED (the shards of one subgraph
                      * run on different ranks, paper_conf_ipps_zhanghl21_b200/multirank.py). */
} duet_partition_opts;

typedef struct {
  int warmup;          /* untimed replays before sampling (default 20)                     */
  int samples;         /* timed samples per subgraph; "e.g., 500" (default 500) */
  int reps_per_sample; /* graph replays between one event pair (default 20)                */
  int calibrate_comm;  /* 1: measure the same-GPU cross-stream alpha (else alpha = 0)      */
} duet_profile_opts;

typedef struct {
  int mode;              /* 0 greedy-correction, 1 greedy only (Steps 1-2),
                            2 serial on the home slot (operators-in-sequence),
                            3 fixed assignment (tests / experiments),
                            the Fig. 13 baselines:
                            4 random, 5 round-robin (slot = id mod D), 6 random + correction */
  int correction_rounds; /* x of "x round of swaps ... without decreasing"; 1 */
  int allow_fallback;    /* 1: best single slot if not slower            */
  const int32_t* fixed_slot_of; /* mode 3: slot per subgraph (length n_sg)                  */
  uint32_t seed;         /* modes 4, 6: slot of s = h(seed, s) mod D, h = lowbias32 of
                            (seed * 0x9E3779B1 + s) mod 2^32 (R-29)               */
} duet_sched_opts;

/* Measured-mode options (duet_schedule_measured). */
typedef struct {
  int samples;          /* timed replays per candidate assignment; latency = lower median; 20  */
  int warmup;           /* untimed replays per candidate before timing; 3                      */
  int64_t measured_ns;  /* OUT: measured latency of the returned assignment                     */
  int32_t evaluations;  /* OUT: distinct assignments captured and timed                         */
} duet_measure_opts;

/* Thread-local message of the last failing call on this thread (valid until the next call). */
const char* duet_last_error(void);
int duet_abi_version(void);

/* ---- graph (PAPER.md:78 input = pre-compiled model; :83 adjacency list) --------------------- */
/* Parse and validate IR text (len bytes, need not be NUL-terminated). */
duet_status duet_graph_load(const char* ir_text, size_t len, duet_graph_t** out);
/* Bind parameter `param` (name without '@') to caller-owned device memory.  dtype/shape must
 * equal the IR declaration; all parameters must be on one GPU. Rebinding replaces the view. */
duet_status duet_graph_bind(duet_graph_t* g, const char* param, const duet_tensor* t);
/* Counts and per-node info (for tests/tools). op_name may be NULL. */
duet_status duet_graph_info(const duet_graph_t* g, int32_t* n_nodes, int32_t* n_inputs,
                            int32_t* n_outputs, int32_t* n_params);
void duet_graph_destroy(duet_graph_t* g);

/* ---- partition (§IV-A) ------------------------------------- */
duet_status duet_partition(const duet_graph_t* g, const duet_partition_opts* o, duet_partition_t** out);
/* Call with NULL arrays to get the counts, then with caller arrays of at least that size:
 *   node_to_sg[n_nodes] (-1 for inputs), sg_phase[n_sg], phase_kind[n_phase] (0 sequential,
 *   1 multi-path), edge_src/dst/bytes[n_edge] in (src,dst) lexicographic order; -1 = graph
 *   input (src) / graph output (dst); bytes = sum over distinct boundary tensors. */
duet_status duet_partition_export(const duet_partition_t* p, int32_t* node_to_sg, int32_t* sg_phase,
                                  uint8_t* phase_kind, int32_t* edge_src, int32_t* edge_dst,
                                  int64_t* edge_bytes, int32_t* n_sg, int32_t* n_phase,
                                  int32_t* n_edge);
/* Row shards of a batch_shards = k partition (PAPER.md:79 phases with
 * the paper's subgraphs split by rows for more devices than branches).  sg_shard[n_sg]: shard
 * index j of each subgraph (rows [j B / k, (j+1) B / k)), -1 if unsharded (sequential phases, or
 * k = 1); sg_origin[n_sg]: the id the subgraph has in the k = 1 partition.  Shards of one subgraph
 * have consecutive ids; node_to_sg maps a sharded node to its shard 0.  A boundary tensor of b
 * bytes entering or leaving shard j carries floor(b (j+1) / k) - floor(b j / k) bytes.  NULL
 * arrays allowed (counts only). */
duet_status duet_partition_shards(const duet_partition_t* p, int32_t* sg_shard, int32_t* sg_origin,
                                  int32_t* n_sg);
void duet_partition_destroy(duet_partition_t* p);

/* ---- profile (§IV-B; 500 runs PAPER.md:87) -------------------------------------- */
/* Time every subgraph's compiled kernels on the device with CUDA events: each sample is the
 * mean of R replays of the subgraph's CUDA graph between one event pair; T = lower median of
 * the samples, int64 ns.  Slots on one GPU share one measurement.  Requires all parameters
 * bound; every slot must be on the parameters' GPU in this build. */
duet_status duet_profile(const duet_partition_t* p, const duet_slot* slots, int n_slots,
                         const duet_profile_opts* o, duet_profile_t** out);
/* Profile from a caller table t_ns[n_sg * n_slots] (row-major by subgraph) — for bit-exact
 * scheduler tests and for replaying a stored profile. */
duet_status duet_profile_from_table(const duet_partition_t* p, int n_slots, const int32_t* slot_gpu,
                                    const int64_t* t_ns, const duet_comm_model* c,
                                    duet_profile_t** out);
/* Any pointer may be NULL. t_ns[n_sg*n_slots], slot_gpu[n_slots]. */
duet_status duet_profile_export(const duet_profile_t* pr, int64_t* t_ns, int32_t* slot_gpu,
                                duet_comm_model* c, int32_t* n_slots);
void duet_profile_destroy(duet_profile_t* pr);

/* ---- schedule (PAPER.md:81, Algorithm 1; fallback PAPER.md:71, :90) ------------- */
duet_status duet_schedule(const duet_partition_t* p, const duet_profile_t* pr, const duet_sched_opts* o,
                          duet_schedule_t** out);
/* Measured mode (Algorithm 1's "measure latency"): the same
 * Steps 1-2 (or random start) from the profile, then Step 3 and the fallback compare candidate
 * assignments by their latency MEASURED on the device: each distinct assignment is captured as
 * the duet_run executor graph over `slots` (device staging buffers filled with synthetic data,
 * no host copies), replayed mo->warmup times, then mo->samples times between CUDA events on
 * slots[0].stream; latency = lower median, int64 ns, memoised per assignment.  Synchronous
 * (blocks the host).  Not deterministic: two calls may return different assignments.  Modes
 * 1..5 have no Step 3 and only measure the fallback.  Requires bound parameters and slots on
 * the parameters' GPU.  mo may be NULL (defaults; no OUT fields). */
duet_status duet_schedule_measured(const duet_partition_t* p, const duet_profile_t* pr,
                                   const duet_sched_opts* o, const duet_slot* slots, int n_slots,
                                   duet_measure_opts* mo, duet_schedule_t** out);
/* Any pointer may be NULL. sg_to_slot[n_sg]; order[n_sg] = global issue order pi (per-slot
 * order = pi filtered by slot); model makespan in ns. */
duet_status duet_schedule_export(const duet_schedule_t* s, int32_t* sg_to_slot, int32_t* order,
                                 int64_t* model_makespan_ns, int32_t* fell_back);
void duet_schedule_destroy(duet_schedule_t* s);

/* ---- run (§IV-D) ---------------------------------------------------------------- */
/* Enqueue one inference on slots[0].stream (asynchronous; no host sync).  The caller orders the
 * home stream after the producers of the inputs (e.g. an event wait) and reads the outputs after
 * the home stream reaches this point.  inputs[] follow the IR's input nodes in declaration order,
 * outputs[] the IR's output nodes in declaration order.  Device tensors are
 * used in place.  HOST tensors must be pinned (page-locked; else DUET_EINVAL).  A host input
 * whose only consumer reads it once, coalesced (hash_mod, the ids of gather_sum / gather_concat),
 * is read by that kernel directly over PCIe (zero-copy); a host output no node consumes, produced
 * by a join / reduce_sum / gather_sum, is stored directly into host memory; other host tensors
 * are copied H2D before / D2H after the graph on the home stream (DUET_ZERO_COPY=0: always copy).
 * Host buffers must stay untouched until the home stream passes this call.  Slot streams other than the home stream only shape
 * the captured CUDA graph (one graph per distinct (slots, tensor pointers) — cached). */
duet_status duet_run(duet_schedule_t* s, const duet_slot* slots, int n_slots, const duet_tensor* inputs,
                     int n_in, duet_tensor* outputs, int n_out);

/* Device trace of the executor (§IV-D: the executor starts a subgraph once its
 * predecessors finish).  With tracing on, later duet_run calls of this schedule record a timing
 * event at the fork and around every subgraph on its slot stream (a separate cached graph; the
 * untraced graph is unchanged).  duet_schedule_trace waits for the last traced run and writes, per
 * subgraph, start_ns[i] / end_ns[i] = its first kernel's start / last kernel's end in ns after the
 * fork (event resolution ~0.5 us); n_sg must equal the partition's subgraph count.  DUET_ESTATE
 * when the last run was not traced.  Either array may be NULL.  tools/trace_json.py writes them
 * as a Chrome trace; tests check start(v) >= end(u) on every partition edge. */
duet_status duet_schedule_set_trace(duet_schedule_t* s, int on);
duet_status duet_schedule_trace(const duet_schedule_t* s, int64_t* start_ns, int64_t* end_ns, int32_t n_sg);

/* Number of kernel launches one duet_run of this schedule performs (for the bench's
 * "gpu_launches" claim).  Valid after the first duet_run. */
duet_status duet_schedule_launch_count(const duet_schedule_t* s, int64_t* n_kernels);

/* ---- kernel-level entry points (parity tests / roofline bench; same kernels as duet_run) ---- */
/* Run node `node_name` of a bound graph alone on `stream`, reading its graph inputs from the
 * given device tensors (in node-argument order of its %-arguments) and writing `out`.  Used to
 * time and check one kernel family in isolation. */
duet_status duet_node_run(duet_graph_t* g, const char* node_name, const duet_tensor* args, int n_args,
                          duet_tensor* out, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* DUET_H_ */
