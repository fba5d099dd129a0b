/*
 * deepplan.h -- C-ABI of the B200-native DeepPlan cold-start hot path.
 *
 * Paper: Jeong, Baek, Ahn, "Fast and Efficient Model Serving Using Multi-GPUs with
 * Direct-Host-Access", EuroSys '23.  Citations "P:<n>" are lines of PAPER.md.
 *
 * DeepPlan "takes a pre-trained DL model as an input", profiles each layer (P:198,
 * §4.3.1), generates an execution plan (Algorithm 1, transmission
 * planning P:227-229) and deploys it to an engine with five execution options --
 * Baseline, PipeSwitch, DHA, PT, PT+DHA -- whose load / migration / execution
 * streams are coordinated by per-layer CUDA events (§4.3.4).  This header
 * exposes exactly those steps.
 *
 * Conventions
 *  - Every function returns dp_status: DP_OK (0) or a negative error code.  On error,
 *    dp_last_error() returns a thread-local message.  No C++ exception crosses the ABI.
 *  - "Device pointer": memory of the named CUDA device (allocated by the caller, e.g.
 *    torch).  "Host pointer": ordinary host memory, read synchronously during the call.
 *  - Streams are passed as void* (a cudaStream_t; NULL = legacy default stream).
 *  - All int64 times are nanoseconds.  Method encoding: DP_LOAD = 0, DP_DHA = 1.
 *  - Thread safety: a dp_context and the models registered with it must be used from one
 *    host thread at a time (the serving harness runs its own worker threads internally).
 */
#ifndef DEEPPLAN_H_
#define DEEPPLAN_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif
#if defined(__GNUC__)
#pragma GCC visibility push(default) /* the library builds with -fvisibility=hidden */
#endif

typedef int32_t dp_status;
#define DP_OK 0
#define DP_ERR_INVALID (-1)     /* bad argument / shape mismatch */
#define DP_ERR_CUDA (-2)        /* a CUDA runtime/driver call failed */
#define DP_ERR_NCCL (-3)        /* an NCCL call failed */
#define DP_ERR_OOM (-4)         /* host (pinned) or device allocation failed */
#define DP_ERR_UNSUPPORTED (-5) /* valid request this build does not implement */
#define DP_ERR_STATE (-6)       /* call not valid in the object's current state */

#define DP_LOAD 0 /* "O": load-then-execute (Table 3 caption) */
#define DP_DHA 1  /* "X": direct-host-access */
#define DP_INF_NS ((int64_t)1 << 50) /* exe_dha_ns of a DHA-ineligible unit */
#define DP_MAX_DEVICES 8

/* Model families of the paper's transformer workloads. */
enum { DP_FAMILY_BERT = 0, DP_FAMILY_ROBERTA = 1, DP_FAMILY_GPT2 = 2 };
/* Weight storage dtypes (the paper never states one; fp16 is the default).  DP_FP32
 * is the paper's own precision (Table 1's byte counts are fp32): every kernel then
 * reads and writes fp32 and the linears run on CUDA cores (there is no fp32 tcgen05 kind). */
enum { DP_FP16 = 0, DP_BF16 = 1, DP_FP32 = 2 };
/* Planning-unit kinds (Table 3: Emb, LN, FC). */
enum { DP_UNIT_EMB = 0, DP_UNIT_LN = 1, DP_UNIT_LINEAR = 2 };
/* Engine options + the "initial approach" of P:41 (GREEDY). */
enum {
  DP_MODE_BASELINE = 0,   /* load every layer, then execute (Fig.1b) */
  DP_MODE_PIPESWITCH = 1, /* per-layer load/execute pipelining, all LOAD (Fig.1c, [6]) */
  DP_MODE_GREEDY = 2,     /* DHA iff Exe(DHA) < Load + Exe(InMem), layer by layer */
  DP_MODE_DHA = 3,        /* Algorithm 1 */
  DP_MODE_PT = 4,         /* parallel transmission, all LOAD (§4.2) */
  DP_MODE_PT_DHA = 5,     /* Algorithm 1 on partition 0 + PT for the rest */
  /* NEXT-row extension, not the paper's (R19): Algorithm 1 on a
   * pipeline model where DHA reads occupy the primary link (cost.dha_link_ns) */
  DP_MODE_DHA_LINK = 6,
  DP_MODE_PT_DHA_LINK = 7,
  /* NEXT-row extension f1(i)+(ii), R20: PT_DHA with the equal split taken over the
   * bytes actually transferred (DHA units count 0) and Algorithm 1 re-run under the PT
   * arrival model on partition 0 */
  DP_MODE_PT_DHA_BAL = 8,
  DP_MODE_PT_DHA_LINK_BAL = 9, /* the same on the link-aware model (R19 + R20) */
  /* NEXT-row extension, R22: instead of contiguous partitions, the loaded units are
   * striped over the k links by earliest arrival at the primary (so the links deliver the
   * model front to back together), with Algorithm 1 run under that PT arrival model */
  DP_MODE_PT_DHA_STRIPE = 10,
  DP_MODE_PT_DHA_LINK_STRIPE = 11 /* the same on the link-aware model (R19 + R22) */
};

/* ---------------------------------------------------------------------------------
 * Errors
 * --------------------------------------------------------------------------------- */
const char* dp_last_error(void);
int32_t dp_abi_version(void); /* 2 (round 2: dp_serve_result / dp_serve_opts / dp_engine_opts fields) */

/* ---------------------------------------------------------------------------------
 * Planner (pure host code, deterministic, no GPU).  §4.3.2-4.3.3, SURVEY §8(c) P1-P4.
 * --------------------------------------------------------------------------------- */

/* Per-unit performance table ("performance table"; Fig.10).
 * All arrays have n entries, caller-owned.  fwd_ns = secondary->primary NVLink time
 * (our addition for PT).  exe_dha_ns = DP_INF_NS marks DHA-ineligible units. */
typedef struct {
  int32_t n;
  const int64_t* bytes;
  const int64_t* load_ns;
  const int64_t* fwd_ns;
  const int64_t* exe_mem_ns;
  const int64_t* exe_dha_ns;
  /* nullable; our NEXT-row extension: time the unit's DHA reads occupy
   * the primary PCIe link (touched bytes / link bandwidth); used only by the *_LINK modes */
  const int64_t* dha_link_ns;
} dp_cost_table;

/* Execution plan: per unit a method (DP_LOAD/DP_DHA) and a slot (0 = the primary GPU's
 * own PCIe link; s >= 1 = PT partition s, forwarded over NVLink).  The plan
 * never names GPUs ("we do not statically assign the GPU"). `serial` = 1 only for
 * DP_MODE_BASELINE (no overlap).  method/slot are caller-owned arrays of n entries. */
typedef struct {
  int32_t n;
  int32_t mode;
  int32_t k; /* number of GPUs whose links carry the model (1 = no PT) */
  int32_t serial;
  int8_t* method;
  int8_t* slot;
} dp_plan;

/* Generate a plan (fills out->method/slot/serial/mode/k; out->n must equal cost->n).
 * DP_ERR_INVALID on n mismatch, k < 1 or k > DP_MAX_DEVICES, unknown mode. */
dp_status dp_plan_generate(const dp_cost_table* cost, int32_t mode, int32_t k, dp_plan* out);

/* Pipeline cost model (the link-aware variant for plan->mode *_LINK): latency,
 * per-unit stall (n entries, nullable) and
 * bytes carried by each link (k entries, nullable). */
dp_status dp_plan_simulate(const dp_cost_table* cost, const dp_plan* plan, int64_t* latency_ns,
                           int64_t* stall_ns, int64_t* link_bytes);

/* Equal-size contiguous partition ("equally partition ... in terms of size"):
 * part[i] = min(k-1, (k * offset_i) / total_bytes).  part: n int8, caller-owned. */
dp_status dp_plan_partition(const int64_t* bytes, int32_t n, int32_t k, int8_t* part);

/* Exhaustive search (optimal under the cost model) over the methods of the `nfree` units
 * listed in free_idx (<= 30), all other units keep base->method; PT partition fixed as in
 * DP_MODE_PT_DHA when base->k > 1 (DP_ERR_INVALID if a free index names a unit of a
 * partition >= 1: those must stay LOAD).  Ties -> lexicographically smallest method vector.
 * out gets the best plan, *latency_ns its latency. */
dp_status dp_plan_exhaustive(const dp_cost_table* cost, const dp_plan* base, const int32_t* free_idx,
                             int32_t nfree, dp_plan* out, int64_t* latency_ns);

/* ---------------------------------------------------------------------------------
 * Context (devices, streams, events, workspaces, peer transport)
 * --------------------------------------------------------------------------------- */
typedef struct dp_context dp_context;

/* devs: CUDA device ordinals usable by this context (1..8).  Creates per device: an
 * execution stream role (the caller's stream is used), `n_h2d` load streams (P:231
 * "load stream"), a migration stream, an event pool. */
dp_status dp_context_create(const int32_t* devs, int32_t ndev, dp_context** out);
dp_status dp_context_destroy(dp_context* ctx);

/* Engine tunables (defaults in brackets).  chunk_bytes: adjacent LOAD units are
 * coalesced into one DMA of up to this many bytes [4 MiB] (one completion event per
 * chunk); n_h2d_streams: load streams per GPU used round-robin [1]; use_graph: capture
 * the cold-start into a CUDA graph per (model, plan, shape, buffers) [0]. */
typedef struct {
  int64_t chunk_bytes;
  int32_t n_h2d_streams;
  int32_t use_graph;
  int32_t gemm_bn;        /* 0 = auto; 32..256 one CTA per tile; -64..-256 CTA pairs (dp_gemm_tc) */
  int32_t debug_delay_us; /* fault injection: stall every load/migration stream this long
                             before each transfer (tests event gating) [0] */
  int32_t debug_poison;   /* 1 = fill HBM slots with 0xFF (NaN) on eviction [0] */
  int32_t use_pdl;        /* chain consecutive kernels with programmatic dependent launch:
                             a kernel's weight prefetch overlaps its predecessor [1] */
  int32_t fuse_ln;        /* 1 = a LayerNorm that follows a resident-weight linear runs in
                             that GEMM's epilogue (a cluster along N exchanges per-token
                             statistics over DSMEM; deterministic; measured slower on B200 at
                             128 tokens) [0] */
  int64_t tail_bytes;     /* the last DMA piece of a link carries at most this many bytes
                             (a unit suffix), so little compute remains after the last byte
                             lands [2 MiB]; 0 = off */
  int32_t persistent;     /* 1 = warm runs execute every layer in ONE persistent kernel (K6: grid =
                             #SMs, grid barriers between ops, next GEMM's weights prefetched under
                             the current op) when all layer units are resident [0] */
  int32_t pt_transport;   /* how a PT slot's units reach the primary:
                             DP_PT_DMA = the secondary's copy engine DMAs each piece over its
                             own PCIe link into a staging ring, then a peer copy (NCCL send/recv
                             across processes) forwards it over NVLink [default];
                             DP_PT_SM = SURVEY f4: a forwarder kernel on the secondary reads
                             the piece from the pinned arena in place (16-byte zero-copy loads
                             over the secondary's PCIe link) and stores it straight into the
                             primary's HBM slot over NVLink -- no staging ring, no second copy;
                             across processes completion is a flag the kernel releases into
                             the primary's memory (dp_peer_ipc_*), not an NCCL call;
                             DP_PT_CE = the same single hop driven by the secondary's copy
                             engine: one DMA per piece from the arena straight into the
                             primary's slot through the peer / IPC mapping (no staging ring) */
  int32_t profile_chain;  /* 1 = dp_profile calibrates the per-unit costs to how the engine runs
                             them (R23): Exe(InMem) rescaled so that their sum is the
                             measured chained warm forward (units timed in isolation -- L2
                             flushed, no PDL overlap -- sum to ~2.6x the real forward on B200;
                             a DHA unit keeps its absolute extra host-read time), and Load = the
                             unit's byte share of one whole-arena copy (the engine coalesces
                             loads, R18; an isolated copy carries ~4 us of per-copy cost) [1] */
  int32_t trace_units;    /* 1 = dp_infer_cold records per-unit timestamps (read back with
                             dp_run_timeline): timing events after every transfer piece and around
                             every unit's dependency wait on the execution stream.  Costs event
                             records between kernels (no PDL overlap) and forces eager enqueue (no
                             graph): a measurement mode [0] */
  int32_t attention_tc;   /* attention core: 0 = by sequence length (K5t, tcgen05 with S, P and O
                             in TMEM, from 384 tokens -- GPT-2 Medium S1024 warm 2.01 -> 1.82 ms --
                             else the mma.sync flash kernels K5 / K5b, faster below 384), 1 =
                             always K5t, 2 = never [0] */
  int32_t reserved[1];
} dp_engine_opts;
#define DP_PT_DMA 0
#define DP_PT_SM 1
#define DP_PT_CE 2
dp_status dp_context_set_opts(dp_context* ctx, const dp_engine_opts* opts);
dp_status dp_context_get_opts(dp_context* ctx, dp_engine_opts* out);

/* Multi-process PT (one process per GPU, P:182 migration over NVLink): every rank
 * calls dp_peer_init with the same 128-byte NCCL unique id (rank 0 creates it with
 * dp_peer_unique_id and the caller distributes it, e.g. via torch.distributed).  The
 * gather uses ncclSend/ncclRecv only.  DP_ERR_NCCL on failure. */
dp_status dp_peer_unique_id(void* out128);
dp_status dp_peer_init(dp_context* ctx, const void* uid128, int32_t rank, int32_t nranks);

/* Multi-process PT without NCCL (opts.pt_transport = DP_PT_SM / DP_PT_CE): records
 * this process's rank among nranks (one device per context).  Either this or dp_peer_init
 * makes dp_infer_cold multi-process: `primary` is then a rank.  With the IPC transports every
 * rank must call dp_infer_cold for every plan with k > 1 (in the same order: the ranks count
 * these cold starts as the epochs of their go / done words); a k = 1 plan is local to the
 * primary.  DP_ERR_STATE if already initialised. */
dp_status dp_peer_init_ipc(dp_context* ctx, int32_t rank, int32_t nranks);

/* Which rank carries each PT slot when `primary` serves (after dp_peer_init[_ipc]; every rank
 * must set the same map): rank_of_slot[s-1] for s = 1..k-1, distinct and != primary.  Without a
 * map slot s is carried by rank (primary + s) mod nranks.  DP_ERR_INVALID on a bad map. */
dp_status dp_peer_set_slot_ranks(dp_context* ctx, int32_t primary, const int32_t* rank_of_slot, int32_t k);

/* ---------------------------------------------------------------------------------
 * Host-link topology (P:148 PCIe-switch contention, P:186 / P:227-229 "GPUs
 * attached to different PCIe switches")
 * --------------------------------------------------------------------------------- */
/* NUMA node of a device's PCI function (sysfs), -1 if unknown. */
int32_t dp_device_numa_node(int32_t dev);
/* NUMA node of the page holding host address p (move_pages), -1 if unknown. */
int32_t dp_host_numa_node(const void* p);
/* Pinned, mapped, portable host memory placed on NUMA node `node` (< 0: no placement): allocated
 * and first-touched by a thread bound to the node's CPUs.  Free with dp_host_free. */
dp_status dp_host_alloc_node(int64_t bytes, int32_t node, void** out);
/* All n devices copy `bytes` host -> device at the same time (each from pinned memory on its own
 * NUMA node), reps times after a warm-up; gbs[i] = device i's median GB/s.  n = 1: the solo rate;
 * n = 2 over (i, j): one entry of the pairwise concurrency matrix. */
dp_status dp_measure_h2d_concurrent(const int32_t* devs, int32_t n, int64_t bytes, int32_t reps, double* gbs);
/* Secondaries for a PT cold start of `primary` over k links, from measured link rates: solo_gbs[n]
 * and pair_gbs[n*n] (device i's rate while j copies concurrently), numa[n] nullable.  Greedy
 * (R25): repeatedly add the GPU that keeps the slowest pairwise-concurrent link of the
 * set fastest; ties -> the primary's NUMA node, then the faster solo link, then the lower index.
 * out: k-1 device indices in slot order.  Pure host code. */
dp_status dp_select_secondaries(const double* solo_gbs, const double* pair_gbs, const int32_t* numa, int32_t n,
                                int32_t primary, int32_t k, int32_t* out);

/* CUDA IPC exchange for the SM forwarder across processes.  dp_peer_ipc_export allocates
 * (once) this rank's HBM slots for `m` and its 16 KiB mailbox (a go word the primary
 * releases at the start of a cold start, and one done word per (slot, piece) the secondaries
 * release when a piece has landed), and writes DP_IPC_HANDLE_BYTES of cudaIpcMemHandle_t
 * data to `out` (caller-owned).  The caller distributes every rank's block (e.g.
 * torch.distributed all_gather); dp_peer_ipc_import takes all nranks blocks concatenated in
 * rank order and opens the other ranks' handles (own block ignored; ranks on the same
 * device are allowed -- loopback across processes).  Both are collective in the sense that
 * every rank calls them for the same model; the handles stay open until dp_model_destroy /
 * dp_context_destroy.  DP_ERR_STATE before dp_peer_init[_ipc]; DP_ERR_CUDA if an IPC call
 * fails. */
#define DP_IPC_HANDLE_BYTES 128
typedef struct dp_model dp_model;
dp_status dp_peer_ipc_export(dp_context* ctx, dp_model* m, void* out);
dp_status dp_peer_ipc_import(dp_context* ctx, dp_model* m, const void* all_handles);

/* ---------------------------------------------------------------------------------
 * Model registration: host weight arena ("we allocate the pinned memory for the
 * layers ... through cudaHostAlloc")
 * --------------------------------------------------------------------------------- */
typedef struct {
  int32_t family;     /* DP_FAMILY_* */
  int32_t vocab, max_pos, type_vocab, hidden, heads, ffn, layers;
  int32_t dtype;      /* DP_FP16 | DP_BF16 */
  int32_t pad_idx;    /* RoBERTa: position ids start at pad_idx + 1 */
  double ln_eps;
} dp_model_config;

typedef struct dp_model dp_model;

typedef struct {
  int32_t kind;          /* DP_UNIT_* */
  int32_t nparams;       /* 1 (embedding) or 2 (weight+bias / gamma+beta) */
  int32_t first_param;   /* index into the parameter list (dp_model_param_info) */
  int32_t reserved;
  int64_t bytes;         /* payload bytes (what a load moves) */
  int64_t arena_offset;  /* byte offset in the arena (256 B aligned) */
  char name[32];         /* e.g. "word", "L3.fc1", "ln_f" */
} dp_unit_info;

typedef struct {
  char hf_name[96];      /* HF state-dict key, e.g. "encoder.layer.0.attention.self.query.weight" */
  int32_t ndim;          /* 1 or 2 */
  int32_t unit;          /* owning unit */
  int64_t shape[2];      /* as the caller supplies it (HF layout; GPT-2 Conv1D is [in,out]) */
  int64_t bytes;
} dp_param_info;

/* Parameter list for a config, BEFORE creating a model (so the caller can marshal by
 * name).  *count gets the number of params; infos (nullable) gets min(cap,count). */
dp_status dp_config_params(const dp_model_config* cfg, dp_param_info* infos, int32_t cap, int32_t* count);

/* Register a model: host_params[i] is a host pointer to parameter i (dp_config_params
 * order) in the storage dtype, row-major, HF layout.  The library COPIES them into its
 * own pinned, mapped, portable arena (GPT-2 Conv1D weights are transposed to [out,in]
 * there) and owns that arena.  DP_ERR_INVALID on bad config; DP_ERR_OOM if pinning fails. */
dp_status dp_model_create(dp_context* ctx, const dp_model_config* cfg, const void* const* host_params,
                          int32_t nparams, dp_model** out);
dp_status dp_model_destroy(dp_context* ctx, dp_model* m);
/* Another instance of the same model (serving, "each instance mimics a model
 * corresponding to a different user"): shares src's pinned arena read-only (freed with the
 * last instance), has its own residency and device state. */
dp_status dp_model_clone(dp_context* ctx, const dp_model* src, dp_model** out);
int32_t dp_model_num_units(const dp_model* m);
dp_status dp_model_unit_info(const dp_model* m, int32_t i, dp_unit_info* out);
int64_t dp_model_bytes(const dp_model* m);
/* Host (mapped) address of the arena, for tests that read it back. */
dp_status dp_model_arena(const dp_model* m, const void** ptr, int64_t* bytes);

/* Transfer schedule of one plan slot (host-only, no GPU): the contiguous pieces (whole
 * units, forward order, <= chunk_bytes unless one unit is larger; the last piece cut down
 * to the longest unit suffix <= tail_bytes) that the slot's link carries -- what
 * dp_infer_cold DMAs on slot 0 and what secondary s sends / the primary receives for
 * slot s >= 1.  Arrays of `cap` entries (nullable); *count = #pieces. */
dp_status dp_transfer_schedule(const dp_model_config* cfg, const dp_plan* plan, int32_t slot, int64_t chunk_bytes,
                               int64_t tail_bytes, int64_t* piece_off, int64_t* piece_bytes, int32_t* first_unit,
                               int32_t* last_unit, int32_t cap, int32_t* count);

/* ---------------------------------------------------------------------------------
 * Profiling (§4.3.1; Table 5).  Per unit, median over `iters`
 * (after 3 warm-ups) of: load_ns (H2D of the unit alone on dev's link), fwd_ns (a peer
 * copy of the unit's bytes; on a 1-GPU context a device-to-device copy), exe_mem_ns /
 * exe_dha_ns (the unit's kernels with its weights in HBM / host-mapped, L2 flushed).
 * out arrays: n entries each (caller-owned; out->n must equal the unit count).
 * --------------------------------------------------------------------------------- */
dp_status dp_profile(dp_context* ctx, dp_model* m, int32_t dev, int32_t batch, int32_t seq, int32_t iters,
                     dp_cost_table* out);

/* Link roofline denominator: best of `reps` H2D copies of `bytes` from memory allocated
 * like the weight arena (pinned, mapped, portable) to device `dev`, in GB/s (1e9 B/s). */
dp_status dp_measure_h2d(int32_t dev, int64_t bytes, int32_t reps, double* gbs);

/* ---------------------------------------------------------------------------------
 * Inference (§4.3.4, Fig.9)
 * --------------------------------------------------------------------------------- */
#define DP_STATS_MAX_UNITS 512
typedef struct {
  int64_t h2d_bytes[DP_MAX_DEVICES];    /* bytes moved host->device over each slot's link
                                           (copy-engine DMAs, or the SM forwarder's reads) */
  int64_t nvlink_bytes[DP_MAX_DEVICES]; /* bytes gathered from slot s into the primary */
  int64_t dha_weight_bytes;             /* weight bytes DHA kernels must read (algorithmic) */
  int32_t n_copies;                     /* DMA operations issued */
  int32_t n_events;                     /* completion events recorded */
  int32_t n_kernels;                    /* kernels launched on the execution stream */
  int32_t n_units;
  float wall_enqueue_us;                /* host time spent enqueuing */
  float reserved[3];
} dp_run_stats;

/* Cold start: the model is NOT resident on `primary`.  Weights are read from the host
 * arena per `plan`: DHA units in place by the DHA kernels; slot-0 LOAD units DMA'd over
 * the primary's link on load streams; slot-s LOAD units via PT over secondaries[s-1]
 * (device ordinals in a single-process context, or NCCL ranks after dp_peer_init; a
 * secondary equal to the primary means loopback: staged and forwarded on one GPU).
 * Execution is enqueued on `stream` (the execution stream); every non-DHA unit's first
 * kernel waits on its load event.  d_ids: int32 [batch*seq] on the primary (ids
 * outside [0, vocab) are clamped, so a bad id never reads past a table in the arena);
 * d_out: [batch*seq*hidden] storage dtype; d_pooled: [batch*hidden] or NULL (BERT/
 * RoBERTa pooler).  On return the work is enqueued (asynchronous); the model is then
 * resident on the primary with the plan's DHA units left in host memory.
 * On a secondary rank (after dp_peer_init) only that rank's transfers are enqueued and
 * d_ids/d_out may be NULL.  DP_ERR_STATE if already resident on the primary. */
dp_status dp_infer_cold(dp_context* ctx, dp_model* m, const dp_plan* plan, int32_t primary,
                        const int32_t* secondaries, int32_t nsec, const int32_t* d_ids, int32_t batch,
                        int32_t seq, void* d_out, void* d_pooled, void* stream, dp_run_stats* stats);

/* Per-unit timeline of the last cold start of m on `dev` run with opts.trace_units = 1 (SURVEY
 * §8(b) "per-unit ready/start/end ns"; dp_run_stats is filled at enqueue time, before any of it
 * happened, so the times are read back here).  Synchronises on that cold start.  All times are ns
 * since the cold start's first event on the execution stream; arrays of n = unit count
 * (caller-owned, each nullable):
 *   ready_ns  when the unit's bytes had landed in HBM (the end of its DMA / forwarded piece; 0 for
 *             a DHA unit, which is read in place; -1 if not observable, e.g. another process's IPC
 *             transfer)
 *   start_ns  when the execution stream passed the unit's dependency wait -- its first
 *             kernel can start
 *   end_ns    when the execution stream reached the next unit (its kernels -- and the
 *             parameterless ops charged to it, SURVEY G1 -- are done); units whose kernels are
 *             grouped (BERT's q/k/v: one launch) end when the group's first kernel starts
 *   stall_ns  start_ns minus when the stream reached the wait: the pipeline stall of P:162-170,
 *             the quantity the simulator (dp_plan_simulate) predicts per unit
 * Units the forward never reached (e.g. the pooler without a pooled output) get -1.
 * DP_ERR_STATE if no traced cold start of m ran on dev. */
dp_status dp_run_timeline(dp_context* ctx, dp_model* m, int32_t dev, int32_t n, int64_t* ready_ns, int64_t* start_ns,
                          int64_t* end_ns, int64_t* stall_ns);

/* Warm inference: the model is resident on dev (DP_ERR_STATE otherwise). */
dp_status dp_infer_warm(dp_context* ctx, dp_model* m, int32_t dev, const int32_t* d_ids, int32_t batch,
                        int32_t seq, void* d_out, void* d_pooled, void* stream, dp_run_stats* stats);

/* GPT-2 tied language-model head ("logits", R14): logits[r][v] =
 * sum_h hidden[r][h] * wte[v][h] for r < rows, fp32, row stride = vocab.  d_hidden: rows
 * vectors of `hidden` storage-dtype elements with row stride ld_hidden (e.g. the last
 * position of every sequence of a forward's d_out: ld_hidden = seq*hidden, d_hidden pointing
 * at token seq-1).  wte is read from HBM when the model is resident on dev with its wte unit
 * loaded, else in place from the pinned host arena (direct-host-access: every byte of the
 * table crosses the link once).  Enqueued on `stream`.  DP_ERR_UNSUPPORTED for
 * BERT/RoBERTa; DP_ERR_INVALID on bad arguments. */
dp_status dp_lm_head(dp_context* ctx, dp_model* m, int32_t dev, const void* d_hidden, int32_t ld_hidden,
                     int32_t rows, float* d_logits, void* stream);

/* Residency: make the model non-resident on dev.  Synchronises the device first; its HBM slot
 * block returns to the context's per-device pool (reused by the next cold start of any model;
 * dp_pool_trim hands free blocks back to the driver).  A model exported with dp_peer_ipc_export
 * keeps its full-arena slots (peers hold IPC mappings of them). */
dp_status dp_model_evict(dp_context* ctx, dp_model* m, int32_t dev);
int32_t dp_model_is_resident(const dp_model* m, int32_t dev);
/* HBM bytes the resident model holds on dev (0 if not resident): only the LOADED units take
 * slots -- a cold start lays the block out like the arena with every DHA unit's range left out,
 * so DHA layers cost no GPU memory ("DeepPlan can serve more instances"). */
int64_t dp_model_resident_bytes(const dp_model* m, int32_t dev);
/* HBM bytes a cold start under `plan` will hold (the compact layout; what the serving harness
 * budgets per instance); -1 on a NULL / mismatched plan. */
int64_t dp_plan_resident_bytes(const dp_model* m, const dp_plan* plan);
/* The per-device slot pool: bytes reserved from the driver and bytes held by resident models. */
dp_status dp_pool_stats(dp_context* ctx, int32_t dev, int64_t* reserved, int64_t* in_use);
/* Release the pool's free blocks to the driver (cudaFree); *freed (nullable) gets the bytes. */
dp_status dp_pool_trim(dp_context* ctx, int32_t dev, int64_t* freed);

/* ---------------------------------------------------------------------------------
 * Kernel entry points (parity-test hooks; same kernels the executor launches).
 * Pointers may be device memory or host memory from dp_host_alloc (mapped) -- the
 * kernels read host memory in place over PCIe (direct-host-access).
 * --------------------------------------------------------------------------------- */
/* Pinned, mapped, portable host memory (cudaHostAlloc) and its release. */
dp_status dp_host_alloc(int64_t bytes, void** out);
dp_status dp_host_free(void* p);

/* SM-driven PT forwarder (the design alternative of P:182): copies `bytes`
 * from `src` (host-mapped pinned memory, read in place with 16-byte loads over the link of
 * the device owning `stream`'s context) to `dst` (device memory of that device or a peer's,
 * written over NVLink) with one kernel; `bytes` may be any size (a sub-16-byte tail is
 * copied bytewise).  src/dst must be 16-byte aligned.  Enqueued on `stream`. */
dp_status dp_pt_forward(const void* src, void* dst, int64_t bytes, void* stream);

/* Embedding: x[t,:] = LN(word[ids[t]] + pos[p(t)] + type[0]) for BERT/
 * RoBERTa (ln_g/ln_b non-NULL), or wte[ids[t]] + wpe[p(t)] for GPT-2 (type, ln NULL).
 * p(t) = pos_offset + (t mod seq).  Every table pointer may be host-mapped (DHA).
 * out_f32 = 1 writes fp32 (the GPT-2 residual stream), else the storage dtype. */
dp_status dp_embed(const int32_t* d_ids, int32_t ntok, int32_t seq, int32_t pos_offset, const void* word,
                   const void* pos, const void* type, const void* ln_g, const void* ln_b, int32_t hidden,
                   double eps, int32_t dtype, int32_t out_f32, void* d_out, void* stream);

/* Linear: y[M,N] = act(x[M,K] w[N,K]^T + b) + residual, row strides ldx/ldy/ldr in
 * elements.  act: 0 none, 1 gelu_erf, 2 gelu_tanh, 3 tanh.  path: 0 = resident tcgen05/
 * TMA GEMM (w must be device memory, N % 128 == 0, K % 64 == 0), 1 = DHA skinny linear
 * (w may be host-mapped; reads every weight byte once).  io: bit0 = residual is fp32,
 * bit1 = y is fp32 (otherwise the storage dtype). */
dp_status dp_linear(const void* x, int32_t ldx, const void* w, const void* b, const void* residual, int32_t ldr,
                    void* y, int32_t ldy, int32_t M, int32_t N, int32_t K, int32_t act, int32_t path, int32_t dtype,
                    int32_t io, void* stream);

/* The resident tcgen05 GEMM of dp_linear(path 0) with its tile configuration forced (tests,
 * sweeps): bn = 0 the cost model's choice; 32/64/96/128/192/256 one CTA per 128 x bn output tile
 * (K2); -64/-128/-192/-256 a CTA pair per 256 x |bn| tile (K2p: cta_group::2 MMAs issued by
 * the even CTA, each CTA staging its 128 W rows and |bn|/2 tokens; needs N % 256 == 0).
 * split = 0 the model's K split, 1 none, 2/4/8 (<= K/64, with a single-CTA bn <= 128) that many
 * K ranges reduced over a thread-block cluster.  Same arguments, layout and errors as
 * dp_linear otherwise; w must be device memory. */
dp_status dp_gemm_tc(const void* x, int32_t ldx, const void* w, const void* b, const void* residual, int32_t ldr,
                     void* y, int32_t ldy, int32_t M, int32_t N, int32_t K, int32_t act, int32_t dtype, int32_t io,
                     int32_t bn, int32_t split, void* stream);

/* LayerNorm over rows of width n: y = LN(x (+ r)) * g + b.  g/b may be host-mapped.
 * x_f32 = 1: x and r are fp32; y is always the storage dtype. */
dp_status dp_layernorm(const void* x, const void* r, const void* g, const void* b, void* y, int32_t rows,
                       int32_t n, double eps, int32_t dtype, int32_t x_f32, void* stream);

/* Attention core: qkv [ntok, 3H] (q | k | v column blocks, row stride ldqkv), heads of
 * d = H/heads (d == 64), softmax(q k^T / sqrt(d) [+ causal mask]) v -> ctx [ntok, H].
 * Sequences are contiguous blocks of `seq` tokens. */
dp_status dp_attention(const void* qkv, int32_t ldqkv, void* ctx_out, int32_t batch, int32_t seq, int32_t hidden,
                       int32_t heads, int32_t causal, int32_t dtype, void* stream);
/* The same on tcgen05 (K5t, the engine's opts.attention_tc): one CTA per (head, 128 queries);
 * S = Q K^T and O_j = P V_j in TMEM, the online softmax per row in one thread, P rounded to the
 * storage type before P.V.  fp16 / bf16, head dim 64, 16-byte aligned rows. */
dp_status dp_attention_tc(const void* qkv, int32_t ldqkv, void* ctx_out, int32_t batch, int32_t seq, int32_t hidden,
                          int32_t heads, int32_t causal, int32_t dtype, void* stream);

/* ---------------------------------------------------------------------------------
 * Serving harness (§5.3): one inference per GPU at a time (Clockwork-like),
 * on-demand cold starts, LRU eviction under a per-GPU byte budget, PT over <= k GPUs.
 * --------------------------------------------------------------------------------- */
typedef struct {
  int64_t arrival_ns; /* offset from trace start */
  int32_t instance;   /* which model instance the request targets */
  int32_t reserved;
} dp_trace_event;

typedef struct {
  int32_t plan_mode;             /* DP_MODE_PIPESWITCH | DP_MODE_DHA | DP_MODE_PT_DHA ... */
  int32_t k_max;                 /* max GPUs per cold start (2 on p3.8xlarge) */
  int32_t ngpu;                  /* GPUs served (dry-run: any; live: <= context devices) */
  int32_t dry_run;               /* 1 = replay with the latency table below, no GPU */
  int64_t per_gpu_budget_bytes;  /* HBM budget for resident instances per GPU */
  int64_t slo_ns;                /* goodput threshold (100 ms) */
  /* dry-run latency table, per MODEL index: cold / warm ns, resident bytes */
  int32_t nmodels;
  int32_t no_prewarm;            /* live: 1 = skip the pre-warm pass (every instance once per GPU) */
  const int64_t* cold_ns;
  const int64_t* warm_ns;
  const int64_t* resident_bytes;
  const int32_t* model_of_instance; /* [ninstances] */
  int32_t ninstances;
  int32_t batch, seq;
  int32_t reserved1;
  /* live mode: models[i] is instance i's dp_model (nmodels == ninstances) and plans[i]
   * its cold-start plan; a plan with k > 1 borrows k-1 other GPUs of the context as
   * secondaries (their PCIe links and copy engines, not their compute): idle ones first.
   * Live decisions are made online on the observed state (R11-live): warm on the
   * GPU holding the instance, else cold on the GPU with the fewest outstanding requests,
   * evicting LRU instances without outstanding requests (dp_model_evict: HBM back to the
   * pool) until the instance's LOADED bytes fit the budget (cold_ns / warm_ns /
   * resident_bytes are not used).  Token ids are 3 + (t * 7919) % 997. */
  const dp_plan* const* plans;
  const int32_t* seq_of_model; /* nullable: per model index sequence length (else `seq`) */
} dp_serve_opts;

typedef struct {
  int64_t start_ns;    /* when the request began executing */
  int64_t finish_ns;   /* completion time (live: when the dispatcher observed it) */
  int32_t gpu;         /* GPU that ran it */
  int32_t cold;        /* 1 = cold start */
  int32_t nevicted;    /* instances evicted to make room */
  int32_t sec_mask;    /* live PT cold start: bit g set = GPU g lent its link (0 otherwise) */
  int64_t decide_ns;   /* live: when the dispatcher decided it (dry run: its arrival) */
} dp_serve_result;

/* Replay (dry_run=1) or run live (dry_run=0: models[] are real dp_models, one per
 * instance, requests are issued at their arrival times on a wall clock).  out: nreq. */
dp_status dp_serve_run(dp_context* ctx, dp_model* const* models, int32_t nmodels, const dp_trace_event* trace,
                       int32_t nreq, const dp_serve_opts* opts, dp_serve_result* out);

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif
#ifdef __cplusplus
}
#endif
#endif /* DEEPPLAN_H_ */
