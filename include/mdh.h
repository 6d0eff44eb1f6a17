/*
 * mdh.h — C-ABI of the B200 (sm_100a) MDH hot path.
 *
 * What this library computes (Schulze, Gorlatch, Rasch, SC-W '25, "Reduction-Aware
 * Directive-Based Programming via Multi-Dimensional Homomorphisms"; PAPER.md = P):
 *
 *   out_view ∘ md_hom[I_1..I_D](f, (⊗_1..⊗_D)) ∘ inp_view          (Listing 7)
 *
 * i.e. for every point i of the index space [0,I_1)×…×[0,I_D) gather the input
 * accesses x(i) = (in_b[ι_{b,a}(i)]) (inp_view), apply the scalar function
 * y(i) = f(x(i)) (md_hom's SF), combine dimension-wise with ⊗_d — cc
 * ("++", places by index, Listing 15) or pw(⊕) (point-wise combine into
 * index 0, Listing 16) — and write R[j] to out_b[ω_{b,a}(j)] (out_view,
 * P:200) with the collapsed (pw) indices equal to 0.  The definition is the
 * footnote-2 formula; every reading of a point the paper leaves open is
 * listed in DESIGN.md §3 (SURVEY §8(c) C-1 … C-29).
 *
 * Conventions (all functions):
 *   - Every function is extern "C", returns mdh_status, never throws.
 *   - Sizes and indices are int64_t.  Buffers are contiguous and row-major
 *     (Listing 1 `M[i*K+k]`); transposes/strides are index functions.
 *   - Device pointers are raw CUDA device pointers (the caller allocates them,
 *     typically as torch tensors).  Host pointers are only taken by
 *     mdh_execute_host and the planning calls.
 *   - Errors: a status code; mdh_last_error() gives a thread-local message that
 *     stays valid until the next mdh_* call on the same thread.
 *   - No CPU fallback exists: every step of mdh_execute runs in this library's
 *     sm_100a kernels; a library built without CUDA support does not exist.
 */
#ifndef MDH_H_
#define MDH_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MDH_ABI_VERSION 3  /* 2: MDH_MAX_ACC 8 -> 32; 3: mdh_stencil_sweeps */

#define MDH_MAX_D     10  /* MCC_Caps is 10-D (Fig 3); configs need <= 7        */
#define MDH_MAX_RANK   8  /* buffer rank                                                */
#define MDH_MAX_ACC   32  /* accesses per buffer (Gaussian_2D 5x5: 25 to one image) */
#define MDH_MAX_BUFS  32  /* PRL: 17 inputs + 3 outputs (Listing 11)         */
#define MDH_MAX_WORLD 64  /* ranks of one multi-GPU plan                                */

typedef enum {
  MDH_OK = 0,
  MDH_ERR_INVALID_ARG = 1,   /* null/misaligned pointer, workspace too small, bad opts  */
  MDH_ERR_INVALID_SPEC = 2,  /* malformed: out-of-bounds access, non-injective output,  */
                             /* size 0, f arity mismatch, declared shape too small      */
  MDH_ERR_UNSUPPORTED = 3,   /* valid MDH but outside this build's catalog: mixed pw    */
                             /* operators (C-3), unknown f/dtype combination, sharding */
                             /* a ps dim                                                */
  MDH_ERR_OUT_OF_MEMORY = 4,
  MDH_ERR_CUDA = 5,          /* a CUDA runtime/driver call or a kernel launch failed    */
  MDH_ERR_NCCL = 6,          /* NCCL missing or an NCCL call failed                     */
  MDH_ERR_INTERNAL = 7
} mdh_status;

/* Basic types (BSC_TYP, Listing 14; Fig 3 "Basic Type" column P:511-531). */
typedef enum {
  MDH_BF16 = 0,  /* bfloat16; accumulated in fp32 (reading C-13/C-15)         */
  MDH_F32 = 1,
  MDH_F64 = 2,
  MDH_I32 = 3,   /* + and * wrap mod 2^32 (reading C-12)                        */
  MDH_U32 = 4,
  MDH_I64 = 5
} mdh_dtype;

/* Combine operators, one per dimension (combine_ops). */
typedef enum {
  MDH_CC = 0,              /* "++" concatenation: index set kept (Listing 15)         */
  MDH_PW_ADD = 1,          /* pw(add)  (Listing 16 with cf = +)                      */
  MDH_PW_MAX = 2,          /* pw(max)                                                */
  MDH_PW_MIN = 3,          /* pw(min)                                                */
  MDH_PW_PRL_ARGMAX = 4,   /* custom pw over the PRL record: lexicographic max of      */
                           /* (id_measure==14, match_weight, match_id); associative and */
                           /* commutative (reading C-19)                                */
  MDH_PW_PRL_PAPER = 5,    /* custom pw, Listing 11 prl_max literally:     */
                           /* res = lhs if lhs.id==14 && rhs.id!=14 else rhs;           */
                           /* associative, NOT commutative — order preserved (C-2)      */
  MDH_PS_ADD = 6           /* ps(add): prefix sum (Listing 17): the dim is   */
                           /* KEPT; result at index k = fold over [0, k] (inclusive),   */
                           /* lhs = lower index range (reading C-25).  May be combined  */
                           /* only with pw(add) dims (MBBS).            */
} mdh_combine;

/* Scalar functions SF ("arbitrary but pure"); a fixed catalog here. */
typedef enum {
  MDH_F_MUL = 0,          /* y = x0 * x1               (f_mul); 2 accesses → 1  */
  MDH_F_STENCIL = 1,      /* y = Σ_a w_a · x_a, w = fparams (reading C-16); n → 1        */
  MDH_F_PRL_COMPARE = 2,  /* Fellegi–Sunter comparison of a (new, db) record pair      */
                          /* (reading C-18): 17 accesses → (match_id i64,             */
                          /* match_weight f64, id_measure i32); fparams = wa[8], wd[8] */
  MDH_F_IDENTITY = 3      /* y = x0; 1 → 1                                             */
} mdh_fn;

/* An affine index function (IDX_FNC; examples P:200-206):
 *   idx[r] = Σ_{d<D} coeff[r][d] · i_d + offset[r],   r < rank   (reading C-8)     */
typedef struct {
  int64_t coeff[MDH_MAX_RANK][MDH_MAX_D];
  int64_t offset[MDH_MAX_RANK];
} mdh_index_fn;

/* A buffer and its accesses (IDF = Buffer[BSC_TYP(,shape)], Listing 12).
 * shape all-zero ⇒ inferred as max accessed index + 1 (fn.7; reading C-9). */
typedef struct {
  mdh_dtype dtype;
  int32_t rank;
  int64_t shape[MDH_MAX_RANK];
  int32_t n_acc;
  mdh_index_fn acc[MDH_MAX_ACC];
} mdh_buffer;

/* The computation (Listing 7 / Listing 14). Dimension d is loop level d (C-26). */
typedef struct {
  int32_t D;
  int64_t size[MDH_MAX_D];      /* I_d >= 1 (reading C-10)                          */
  mdh_combine op[MDH_MAX_D];    /* ⊗_d                                              */
  mdh_fn f;
  int32_t n_fparams;
  const double* fparams;        /* host; copied at plan time                        */
  int32_t n_in;
  const mdh_buffer* in;         /* host array of n_in buffers; accesses in (b,a) order */
  int32_t n_out;
  const mdh_buffer* out;
} mdh_spec;

#define MDH_PLAN_VIRTUAL_SHARD 0x1u  /* plan rank r of world_size on one GPU, no comm */
#define MDH_PLAN_NO_COLLECTIVE 0x2u  /* pw shard: leave the partial result local       */
#define MDH_PLAN_FLOAT_ALLREDUCE 0x4u /* pw(add) shard of a float output: ncclAllReduce
                                        (NVLS in-switch reduction where NCCL selects it)
                                        instead of allgather + ordered combine — faster
                                        for large outputs (split-K MatMul / MCC across
                                        GPUs), but the summation order
                                        is NCCL's: reproducible only for a fixed NCCL
                                        algorithm and topology                          */

typedef struct {
  int32_t device;        /* CUDA device ordinal the plan executes on                   */
  int32_t world_size;    /* 1 ⇒ single GPU                                             */
  int32_t rank;
  void* nccl_comm;       /* from mdh_comm_init, or NULL (VIRTUAL_SHARD / world 1)       */
  int32_t shard_dim;     /* -1 ⇒ the planner chooses (world_size > 1).  world_size 1
                            with nccl_comm and shard_dim >= 0: a one-rank shard that runs
                            the sharded execute path (collective over the one-rank
                            communicator) — the NCCL data plane on one GPU              */
  uint32_t flags;
  const char* tile_table;/* path of a tile table JSON; NULL ⇒ $MDH_TILE_TABLE, else the */
                         /* table compiled into the library                             */
  const char* force_tile;/* "key=value,…" override (like $MDH_FORCE_TILE) or NULL       */
} mdh_plan_opts;

typedef struct mdh_plan_s* mdh_plan_t;

/* Validate `spec`, classify dimensions, choose a kernel template and its tiles, and
 * (world_size > 1) rewrite the spec to this rank's sub-domain.  Host-only work: no
 * device memory is touched except small plan-owned constants (uploaded lazily on the
 * first execute).  Ownership: the plan copies everything it needs from `spec`.
 * Errors: INVALID_SPEC / UNSUPPORTED as described above; INVALID_ARG for bad opts. */
mdh_status mdh_plan(const mdh_spec* spec, const mdh_plan_opts* opts, mdh_plan_t* plan_out);

/* Device workspace the caller must pass to mdh_execute (bytes, 256-B aligned start).
 * The workspace must be ZERO-FILLED before its first use with a plan (e.g. one
 * cudaMemsetAsync); every mdh_execute leaves it zero-filled again where it matters
 * (the cross-CTA combine tickets reset themselves), so it can be reused without
 * re-initialisation.  One workspace must not be used by two concurrent executes. */
mdh_status mdh_plan_workspace_size(mdh_plan_t plan, size_t* bytes);

/* The shape of input (is_output=0) or output (is_output=1) buffer `buf` as THIS rank
 * holds it, and the global coordinates of its element 0.  world_size 1 ⇒ the global
 * (declared or inferred) shape and zeros.  shape/global_offset: host arrays of
 * MDH_MAX_RANK; entries >= rank are 0.  *dtype and *rank may be NULL.              */
mdh_status mdh_plan_local_shape(mdh_plan_t plan, int32_t is_output, int32_t buf,
                                int64_t* shape, int64_t* global_offset,
                                int32_t* dtype, int32_t* rank);

/* A JSON description of the plan (template, tiles, dimension groups, shard).  Writes
 * at most `cap` bytes including the terminating NUL; *needed (may be NULL) gets the
 * full length + 1. */
mdh_status mdh_plan_describe(mdh_plan_t plan, char* json, size_t cap, size_t* needed);

/* Enqueue the computation on `cuda_stream` (a cudaStream_t; NULL = legacy default).
 *   in[b]  : device pointer of input buffer b (local shape), 16-B aligned
 *   out[b] : device pointer of output buffer b, 16-B aligned
 * Semantics: overwrites every output element in the image of the output index
 * functions and leaves all others untouched ("=" not "+="; C-5, C-6);
 * outputs need no initialisation and are never read; inputs must not alias outputs
 * (C-27).  Asynchronous: kernel faults surface at the caller's synchronisation
 * unless MDH_DEBUG_SYNC=1.  Deterministic: no float atomics; repeated runs are
 * bit-identical.  With world_size > 1 and a pw shard dim the NCCL collective and
 * the ordered local combine are enqueued on the same stream.                      */
mdh_status mdh_execute(mdh_plan_t plan, const void* const* in, void* const* out,
                       void* workspace, size_t workspace_bytes, void* cuda_stream);

/* End-to-end variant: in/out are HOST pointers (pinned for full PCIe bandwidth).
 * `device_scratch` (>= mdh_plan_host_scratch_size bytes) holds the device copies and
 * the workspace.  Enqueues H2D copies, the computation and D2H copies on the stream;
 * the caller synchronises before reading `out`.
 * Pipelined (world-size-1 plans with >= 32 MB of host data, $MDH_HOST_PIPE_MIN_MB; off
 * with MDH_HOST_PIPE=0; $MDH_HOST_PIPE_CHUNKS chunks, default 4 — MatMul 4096³ e2e
 * 66.2 / 67.2 / 65.7 TFLOP/s at 4 / 8 / 16): when a cc dim d exists on which every buffer depends only
 * through its coordinate 0 (MatMul rows, Jacobi planes, MCC images, PRL new records),
 * the problem runs as 4 chunks along d (virtual shards of the plan): chunk c's input
 * slices are copied on an internal copy-in stream, computed on `cuda_stream`, and its
 * output slice copied back on an internal copy-out stream, so both PCIe directions and
 * the kernels overlap; inputs that do not depend on d are copied once.  The stream
 * semantics are unchanged: the call's work is ordered after earlier work on
 * `cuda_stream` and later work on it waits for the last D2H copy.  Host output
 * elements outside the output image (C-5) are unspecified after the call.
 * Errors: as mdh_execute; INVALID_ARG for NULL pointers or too little scratch.        */
mdh_status mdh_plan_host_scratch_size(mdh_plan_t plan, size_t* bytes);
mdh_status mdh_execute_host(mdh_plan_t plan, const void* const* host_in,
                            void* const* host_out, void* device_scratch,
                            size_t scratch_bytes, void* cuda_stream);

/* Ordered ⊗-fold of S partial results of this plan (e.g. the per-rank results of a
 * pw shard, in rank = index order): out = p_0 ⊗ p_1 ⊗ … ⊗ p_{S-1} per output element
 * (Listing 16 applied S-1 times, lhs = lower index range).  partial_outs[s*n_out+b]
 * is partial s of output buffer b (device, local output shape).  Only valid for
 * plans whose reduction dims are all the same pw operator.                        */
mdh_status mdh_combine_partials(mdh_plan_t plan, const void* const* partial_outs,
                                int32_t S, void* const* out, void* cuda_stream);

mdh_status mdh_destroy(mdh_plan_t plan);

/* ---- Stencil time-stepping with a halo exchange (reading C-34).
 * The paper evaluates one Jacobi sweep; time-stepping applies the same md_hom
 * repeatedly: sweep t reads buffer src_t and writes dst_t (u→v, v→u, …).
 *
 * `plan` must be an all-cc map with one input and one output buffer of the same dtype and
 * the same shape [nz, …] (e.g. mdh_workloads.specs.jacobi3d_sweep, whose output index
 * function is the input's centre access): its output image is the interior, the rest of
 * the output buffer (the boundary shell) is never written (C-5), so u and v must both
 * hold the fixed boundary on entry.  Buffer dim 0 is the sharded dim: plane = the
 * product of the other extents; the stencil may reach at most one plane below / above
 * (halo width 1).  With halo == NULL or world == 1 this is the whole domain.  Otherwise
 * this rank owns local planes 1..nz-2 of a z-slab, plane 0 / nz-1 being halo copies of
 * the lower / upper neighbour's last / first owned plane; after every sweep the first and
 * last owned planes of dst go to the neighbours' halo planes of their dst:
 *   - NCCL transport (nccl_comm from mdh_comm_init; one process per GPU): grouped
 *     ncclSend/ncclRecv on `cuda_stream`, any number of sweeps per call;
 *   - peer transport (nccl_comm NULL): the neighbours' halo planes peer_lo / peer_hi are
 *     device addresses this process can write (same device, P2P or CUDA-IPC mapped); the
 *     7-point kernel stores its first / last output plane into them itself (compute and
 *     exchange in one kernel), other stencils are followed by device-to-device copies.
 *     The caller orders the ranks' calls (one sweep per call, lock-step — e.g. virtual
 *     ranks on one stream).
 * `workspace` as for mdh_execute.  On return *result_in_v = sweeps odd (the final field
 * is in v), else 0 (in u).  Errors: MDH_ERR_INVALID_ARG (bad plan shape, aliasing u/v,
 * sweeps < 0, missing transport, nz < 3), MDH_ERR_NCCL, MDH_ERR_CUDA.                  */
typedef struct mdh_halo {
  void* nccl_comm;    /* NCCL transport, or NULL                                        */
  int32_t rank;       /* this slab's index along dim 0 (neighbours rank-1, rank+1)      */
  int32_t world;      /* number of slabs                                                */
  void* peer_lo[2];   /* peer transport: lower neighbour's TOP halo plane in its u [0] and v [1] (NULL at rank 0)   */
  void* peer_hi[2];   /* peer transport: upper neighbour's BOTTOM halo plane in its u and v (NULL at rank world-1) */
} mdh_halo;

mdh_status mdh_stencil_sweeps(mdh_plan_t plan, void* u, void* v, int32_t sweeps, const mdh_halo* halo,
                              void* workspace, size_t workspace_bytes, void* cuda_stream,
                              int32_t* result_in_v);

/* NCCL communicator bootstrap (NCCL is loaded with dlopen on first use).
 * id128: 128 bytes (ncclUniqueId) produced on one rank and broadcast by the caller. */
mdh_status mdh_comm_unique_id(void* id128);
mdh_status mdh_comm_init(const void* id128, int32_t world, int32_t rank, int32_t device,
                         void** comm_out);
mdh_status mdh_comm_destroy(void* comm);

const char* mdh_last_error(void);
int32_t mdh_abi_version(void);

/* Number of kernel launches the last mdh_execute/mdh_execute_host/mdh_combine_partials
 * on this thread enqueued (for the bench's gpu_launches claim).                     */
int32_t mdh_last_launch_count(void);

/* Diagnostics only (not part of the computation): with MDH_T4_TRACE=1 in the environment
 * the T4 2-SM tensor-core kernel records, per work unit u of its last launch, eight u64 at
 * host[8u..8u+7]: (SM id << 32 | CTA-pair id, %globaltimer ns at the unit's first MMA
 * issue, at its last MMA commit, at the end of its epilogue, SM cycles the MMA issuer
 * waited for loaded stages, SM cycles it waited for a free accumulator, %globaltimer when a
 * stream-K finisher saw all its partials, when a producer published its partial; else 0).  When
 * all n traced units fit (n ≤ max_units), 1024 more u64 follow at host[8n..]: per CTA pair
 * p < 256 and CTA r of the pair, %globaltimer at kernel entry [2p + 512r] and exit
 * [2p + 1 + 512r]; `host` must then hold 8·max_units + 1024 u64.  Synchronises the device,
 * returns n; 0 when tracing is off, -1 on a CUDA error.  `host` is caller-owned.         */
int64_t mdh_debug_t4_trace(uint64_t* host, int64_t max_units);

/* Diagnostics: measured instruction-throughput peaks of `device` (the roofline
 * denominators of the pipe-bound templates): fp32 FFMA TFLOP/s (8 FFMA
 * chains per thread), ALU-pipe thread-instructions/s (LOP3 chains) and the issue rate
 * (thread-instructions/s: the best of the FFMA kernel and an FFMA/LOP3 interleave) — each
 * the best of 3 ~ms launches
 * of 4 × 256 threads per SM, timed with CUDA events.  Synchronises; any pointer may be
 * NULL.  Errors: MDH_ERR_CUDA.                                                          */
mdh_status mdh_measure_peaks(int32_t device, double* ffma_tflops, double* alu_tops, double* issue_tops);

#ifdef __cplusplus
}
#endif
#endif /* MDH_H_ */
