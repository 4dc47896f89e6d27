/* mggcn.h — C ABI of the B200-native MG-GCN hot path.
 *
 * MG-GCN: Balın, Sancak, Çatalyürek, "MG-GCN: A Scalable multi-GPU GCN
 * Training Framework", ICPP '22.  The paper text is /root/reference/PAPER.md
 * at build time and is cited here as P:line.  The library computes full-batch
 * GCN training on a randomly permuted, 1D row-partitioned
 * graph:
 *     forward   H' = ReLU(Â^T · H · W)                 (Eq. 1, 5-7)
 *     loss      softmax cross-entropy
 *     backward  Eq. 8-11
 *     update    W_G summed over ranks, Adam
 * where Â_uv = A_uv / sum_w A_wv is the in-degree normalised adjacency (Eq. 2,
 * P:312-318).  Every sparse aggregation runs as P stages (Fig. 2-3):
 * the next feature block is broadcast into BC1/BC2 on the communication stream
 * while the current stage's CSR block SpMM runs on the compute stream
 * (§4.3).
 *
 * Conventions (all functions):
 *  - return an int status; 0 = MGGCN_OK.  Nothing throws across the ABI.
 *    mggcn_last_error() returns a thread-local message for the last non-OK
 *    return of the calling thread.
 *  - host inputs are copied before the call returns; the caller may free them.
 *  - device memory is never allocated by the library outside the caller-owned
 *    workspace given to mggcn_model_create (the debug_* test entry points and
 *    the 16-byte buffer of the NCCL start-up self-check are the exceptions).
 *  - all matrices are row-major fp32; W_l is d_l x d_{l+1} (so H·W is Eq. 5).
 *  - CUDA / NCCL errors poison a model: every later call on it returns the
 *    same code.
 *  - multi-GPU models (NCCL or MGGCN_F_IPC): every host wait (forward with a
 *    loss, the get_* getters, profile / timeline reads, mggcn_model_free)
 *    polls ncclCommGetAsyncError and gives up after MGGCN_SYNC_TIMEOUT_S
 *    seconds (environment, default 600): a failed collective or a peer that
 *    never arrives returns MGGCN_ENCCL (communicators aborted) instead of
 *    hanging; mggcn_step polls the async error without waiting.
 *    mggcn_model_create verifies a fresh communicator with one all-reduce and
 *    one broadcast of known values (ENCCL if they come back wrong).
 *  - a model is single-threaded.  Results are bitwise reproducible run to run
 *    for fixed inputs, P and seed (no floating-point atomics); they are NOT
 *    bitwise equal across different P.
 */
#ifndef MGGCN_H
#define MGGCN_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
    MGGCN_OK = 0,
    MGGCN_EINVAL = -1,        /* invalid argument (see each function)              */
    MGGCN_ENOMEM = -2,        /* host allocation failed / workspace too small      */
    MGGCN_ECUDA = -3,         /* CUDA runtime error (model poisoned)               */
    MGGCN_ENCCL = -4,         /* NCCL error (model poisoned)                       */
    MGGCN_ESTATE = -5,        /* call out of order (backward before forward, ...)  */
    MGGCN_EUNSUPPORTED = -6   /* valid but not implemented         */
};

/* Model flags. */
enum {
    MGGCN_F_OVERLAP = 1u,     /* overlap broadcast i+1 with SpMM i.  Off =
                                 each broadcast waits for the previous stage.          */
    MGGCN_F_RELU_LAST = 2u,   /* ReLU on the last layer too (literal Eq. 4, reading C4) */
    MGGCN_F_TF32X1 = 4u,      /* 1xTF32 GEMMs (faster, ~1e-3 rel. error); default is
                                 3xTF32 (hi/lo split, ~fp32 accuracy)                  */
    MGGCN_F_NO_BCAST = 16u,   /* TIMING ONLY: skip broadcasts; results invalid.  With
                                 P > 1, nlocal = 1, nccl_id128 = NULL and no IPC it is
                                 the SOLO mode: one rank of a P-way run alone, every
                                 collective skipped (per-rank compute time of a
                                 partition too large for loopback). */
    MGGCN_F_PROFILE = 32u,    /* record per-op CUDA events (see mggcn_get_profile)     */
    MGGCN_F_NO_COALESCE = 64u,/* keep duplicate entries as separate gathers (default:
                                 merged on the device copy, value = multiplicity)       */
    MGGCN_F_CACHE_L0 = 128u,  /* X is constant across epochs (full-batch training): layer 0
                                 runs SpMM-first and T0 = Â'^T X is computed on the first
                                 forward and reused (exact by associativity,
                                 Eq. 5-6 and Eq. 10).  mggcn_reset_cache() after X changes. */
    MGGCN_F_IPC = 256u,       /* nlocal = 1, P > 1 without NCCL: peers map each
                                 other's workspaces (CUDA IPC, mggcn_ipc_export / _connect);
                                 each receiver PULLS the broadcast blocks with copy engines in
                                 rotated order (no SMs taken from the SpMM), W_G and the loss
                                 scalars are summed in rank order over peer memory, and
                                 cross-process order uses device sequence flags written and
                                 awaited by stream memory operations.  All ranks must issue
                                 the same sequence of calls with the same kind of X argument
                                 (host / device / prefetch); device X is always copied. */
    MGGCN_F_REPL2 = 512u,     /* 1.5D partitioning with replication factor c = 2 (
                                 §5.1, the 1.5D algorithm of the paper's ref [35]).
                                 The parts are P'-way partitions (P' even) and the job has
                                 2P' ranks: rank (i, r) = r * P' + i holds row block i of Â'
                                 and H (every block twice), computes the partial SpMM over the
                                 column blocks j with j mod 2 = r (P'/2 stages; block j is
                                 broadcast inside replica group r only, so each rank receives
                                 n d / 2 values per SpMM instead of (P-1)/P n d), then the two
                                 replicas of a row block sum their partials (pair all-reduce)
                                 and apply the row scale / ReLU.  Only the ROOT replica of a
                                 row block (r = i mod 2, the one that broadcasts it) computes
                                 its GEMM products (H W, the input gradient) and contributes
                                 W_G, the loss and |T|; the other replica adds zeros.
                                 Loopback: nlocal = 2P', parts[k] = part k mod P' (replica
                                 k / P').  NCCL: nlocal = 1, nccl id shared by all 2P'
                                 processes, MGGCN_F_REPLICA1 on the replica-1 processes.
                                 Not with MGGCN_F_IPC (EUNSUPPORTED). */
    MGGCN_F_REPLICA1 = 1024u, /* with MGGCN_F_REPL2 and nlocal = 1: this process is replica 1 */
    MGGCN_F_TIMELINE = 2048u  /* record one CUDA event pair per op on the stream it runs on,
                                 tagged with the SpMM index and stage (the per-stage
                                 comm / compute timelines of Fig. 6 / Fig. 8, P:1372-1403,
                                 P:1545-1580); read with mggcn_get_timeline */
};

/* Size of one rank's IPC descriptor (mggcn_ipc_export). */
#define MGGCN_IPC_BLOB_BYTES 128

typedef struct mggcn_graph_s* mggcn_graph; /* host CSR of A + in-degrees                     */
typedef struct mggcn_part_s* mggcn_part;   /* one rank's permuted 1D partition (host)        */
typedef struct mggcn_model_s* mggcn_model; /* weights, Adam state, buffer plan, comm, streams */

const char* mggcn_last_error(void);
int mggcn_version(void); /* MAJOR*10000 + MINOR*100 + PATCH */

/* ------------------------------------------------------------------ ingest
 * mggcn_load_csr — the adjacency A in R^{n x n} as CSR.
 *   rowptr  int64[n+1], host; rowptr[0] = 0, non-decreasing, rowptr[n] = nnz
 *   colidx  int32[nnz], host; in [0, n); any order within a row
 *   vals    fp32[nnz] host, finite and > 0; NULL means A_uv = 1 (pattern-only)
 *   Duplicate entries are multiplicities (reading C19).  Computes the
 *   weighted in-degree deg(v) = sum_u A_uv (fp64 in CSR order, rounded to
 *   fp32; Eq. 2, reading C18) and detects multiset symmetry.
 *   EINVAL: n <= 0, n >= 2^31, malformed rowptr, colidx out of range, bad vals. */
int mggcn_load_csr(int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx, const float* vals,
                   mggcn_graph* out);
/* n, nnz, symmetric (0/1), unit weights (0/1); deg: fp32[n] host or NULL. */
int mggcn_graph_info(mggcn_graph g, int64_t* n, int64_t* nnz, int32_t* symmetric, int32_t* unit_weights,
                     float* deg);

/* --------------------------------------------------------------- partition
 * mggcn_partition — random vertex permutation pi (splitmix64
 * Fisher-Yates from perm_seed, reading C15; 0 = identity), uniform partition
 * vector p(i) = floor(i n / P) (Eq. 13, reading C14), and for `rank` the P
 * forward tiles F_rank,j (rows p(rank)..p(rank+1)-1 of Â'^T restricted to
 * columns p(j)..p(j+1)-1, local indices, Eq. 14-15) and backward tiles
 * B_rank,j (the same rows of Â').  Pure host work.
 *   nparts in [1, 64], rank in [0, nparts), n >= nparts.
 *   EUNSUPPORTED: a tile with >= 2^31 entries. */
int mggcn_partition(mggcn_graph g, int32_t nparts, int32_t rank, uint64_t perm_seed, mggcn_part* out);
/* p: int64[P+1] or NULL; perm: int64[n] (perm[old] = new) or NULL;
 * tile_nnz: int64[2P] (F_rank,0..P-1 then B_rank,0..P-1) or NULL. */
int mggcn_part_info(mggcn_part part, int32_t* nparts, int32_t* rank, int64_t* n, int64_t* p, int64_t* perm,
                    int64_t* tile_nnz);
/* Host copy of tile (dir 0 = forward F_rank,j of Â'^T, 1 = backward B_rank,j
 * of Â'): rowptr int32[n_rank+1], colidx int32[nnz], vals fp32[nnz] (the
 * value Â'_uv of every entry; may be NULL).  Bit-exact test contract. */
int mggcn_part_export_tile(mggcn_part part, int32_t dir, int32_t j, int32_t* rowptr, int32_t* colidx, float* vals);
/* inv_deg of this rank's rows (fp32 1/deg, 0 when deg = 0, reading C20). */
int mggcn_part_inv_deg(mggcn_part part, float* inv_deg);

/* ------------------------------------------------------------------- model
 * dims: int32[L+1] = d_0 .. d_L (d_0 = input features, d_L = classes).
 * parts: nlocal partitions.  nlocal = 1 is the production mode (one process
 * per GPU; for P > 1, nccl_id128 is the ncclUniqueId from
 * mggcn_nccl_unique_id on rank 0, shared by the caller, e.g. through
 * torch.distributed).  nlocal = P (parts for ranks 0..P-1 in order,
 * nccl_id128 = NULL) is the LOOPBACK mode: all P ranks live on the current
 * device and broadcasts become device copies with the identical event
 * schedule (test harness for the P-stage pipeline on one GPU).
 * workspace: device memory, caller-owned, >= mggcn_workspace_bytes, 256-B
 * aligned; it must outlive the model.  compute_stream / comm_stream:
 * cudaStream_t values (streams 0 and 1 of P:929-933); 0 = legacy default.
 * With NCCL (P > 1) and MGGCN_F_OVERLAP the SpMM launches oversubscribed grids
 * whose blocks retire throughout the launch, so NCCL's kernels can take SMs
 * mid-stage: give comm_stream the higher priority (cudaStreamCreateWithPriority).
 * EUNSUPPORTED: an SpMM-first layer (d_l < d_{l+1}) at l > 0. */
int mggcn_workspace_bytes(const mggcn_part* parts, int32_t nlocal, int32_t L, const int32_t* dims, uint32_t flags,
                          size_t* bytes);
int mggcn_model_create(const mggcn_part* parts, int32_t nlocal, int32_t L, const int32_t* dims, uint32_t flags,
                       const void* nccl_id128, void* workspace, size_t ws_bytes, uintptr_t compute_stream,
                       uintptr_t comm_stream, mggcn_model* out);
int mggcn_nccl_unique_id(void* out128);
/* MGGCN_F_IPC models (P > 1, nlocal = 1, nccl_id128 = NULL): every rank calls
 * mggcn_ipc_export (writes MGGCN_IPC_BLOB_BYTES host bytes: the CUDA IPC
 * handle of the allocation that holds its workspace + the offset, rank, P and
 * symmetric-region size), the caller exchanges the P blobs (e.g. all_gather over
 * torch.distributed), then every rank calls mggcn_ipc_connect with the P blobs
 * in rank order (host, P * MGGCN_IPC_BLOB_BYTES bytes), which maps the peers'
 * workspaces (cudaIpcOpenMemHandle; unmapped by mggcn_model_free).  The
 * workspace must then stay allocated in every process until all models are
 * freed.  EINVAL: not an IPC model, blobs of another P / plan / rank order, or
 * connect called twice; ECUDA: the IPC calls failed (e.g. no P2P between the
 * devices); ESTATE from mggcn_forward until connected. */
int mggcn_ipc_export(mggcn_model m, void* blob);
int mggcn_ipc_connect(mggcn_model m, const void* blobs);

/* Weights W_l (d_l x d_{l+1}, host fp32).  set_weights resets Adam (t = 0). */
int mggcn_set_weights(mggcn_model m, int32_t layer, const float* W);
int mggcn_get_weights(mggcn_model m, int32_t layer, float* W);

/* ----------------------------------------------------------- the hot path
 * mggcn_forward — L layers (Eq. 5-7 with the §4.4 order rule), then the
 * softmax-CE loss and its gradient (written in place, Eq. 19).
 *   X_local  fp32 rows of X' owned by this model (rows p(rank)..p(rank+1)-1
 *            of the PERMUTED features; all n rows in loopback mode), row
 *            stride ldx >= d_0.  Host or device pointer (host: copied on the
 *            compute stream; this is the end-to-end path).  A device X whose
 *            stride is the library's padded ld (d_0 rounded up to 8) and that
 *            is 16-B aligned is read IN PLACE (no copy): it must then stay valid
 *            and unchanged until this epoch's mggcn_backward has completed.
 *            A host X with the padded stride is copied with one contiguous
 *            copy (fastest end-to-end path); any other stride goes through
 *            a device staging chunk.  Padding columns are never read as data.
 *            NULL: use the inputs of the pending mggcn_prefetch.
 *   y_local  int32 labels of the same rows (host or device); -1 = unlabelled.
 *   loss     host out: global mean CE over labelled vertices (reading C5), or
 *            NULL (no host synchronisation).
 *   logits_local  device out (n_local x d_L, ld = d_L) or NULL.
 * mggcn_backward — Eq. 8-11 for l = L-1..0, per-layer W_G all-reduce
 *   (P:696-704).  ESTATE without a prior forward.
 * mggcn_step — waits for the W_G all-reduce, Adam (reading C6), t++.
 *   ESTATE without a prior backward. */
int mggcn_forward(mggcn_model m, const float* X_local, int64_t ldx, const int32_t* y_local, float* loss,
                  float* logits_local);
int mggcn_backward(mggcn_model m);
/* mggcn_prefetch — enqueue the host->device copy of the NEXT forward's inputs
 * (same arguments as mggcn_forward) on a library-owned copy stream into the
 * second input buffer, so that it overlaps the current epoch; the next
 * mggcn_forward(m, NULL, 0, NULL, ...) consumes it.  The caller keeps the
 * host buffers valid until that forward returns.  ESTATE if one is pending. */
int mggcn_prefetch(mggcn_model m, const float* X_local, int64_t ldx, const int32_t* y_local);
/*   EUNSUPPORTED with MGGCN_F_IPC when layer 0 is SpMM-first (X itself is exchanged: the peers
 *   pull it from this rank's current input buffer, so every rank must use the same one; X is
 *   then also always copied into the workspace, never used in place). */
/* Drops the MGGCN_F_CACHE_L0 aggregate; the next forward recomputes it from X. */
int mggcn_reset_cache(mggcn_model m);
int mggcn_step(mggcn_model m, float lr, float beta1, float beta2, float eps);

/* ------------------------------------------------------- captured epochs
 * mggcn_epoch_capture — records ONE whole epoch (mggcn_forward with loss =
 *   NULL and no logits -> mggcn_backward -> mggcn_step(lr, beta1, beta2, eps))
 *   on the compute stream into a CUDA graph; nothing executes.  The epoch is
 *   Fig. 1's forward / loss / backward / Adam sequence with the
 *   same kernels, streams and events as the eager calls; the comm stream is
 *   forked and joined inside the graph.  X_local / y_local: DEVICE pointers
 *   (same meaning as in mggcn_forward) whose addresses the graph bakes in:
 *   each replay reads whatever they hold then, so the caller keeps them valid
 *   and may refill them between replays.  Only between epochs (ESTATE after
 *   a forward/backward without step or with a prefetch pending); EINVAL for
 *   host pointers; EUNSUPPORTED with MGGCN_F_IPC or MGGCN_F_CACHE_L0, or if
 *   the stream cannot be captured.  A new capture replaces the old graph;
 *   mggcn_model_free releases it.
 * mggcn_epoch_replay — launches the captured epoch `epochs` times on the
 *   compute stream (asynchronous).  Adam's step count advances per replay
 *   (its bias corrections are re-set in the graph before each launch), so N
 *   replays are bitwise the same as N eager epochs.  mggcn_get_loss reads the
 *   last replay's loss.  ESTATE without a capture or mid-epoch. */
int mggcn_epoch_capture(mggcn_model m, const float* X_local, int64_t ldx, const int32_t* y_local, float lr,
                        float beta1, float beta2, float eps);
int mggcn_epoch_replay(mggcn_model m, int32_t epochs);

/* Synchronising getters / checkpoint. */
int mggcn_get_loss(mggcn_model m, float* loss);                 /* loss of the last forward */
int mggcn_get_grad(mggcn_model m, int32_t layer, float* WG);    /* reduced W_G of the last backward */
int mggcn_get_adam(mggcn_model m, int32_t layer, float* mom, float* vel, int64_t* t);
int mggcn_set_adam(mggcn_model m, int32_t layer, const float* mom, const float* vel, int64_t t);

/* Profiling (MGGCN_F_PROFILE): accumulated device milliseconds and launch
 * counts per op class since the last reset, measured with CUDA events on the
 * stream each op is launched on.  Classes: 0 spmm, 1 gemm, 2 loss, 3 adam,
 * 4 bcast, 5 allreduce, 6 other, 7 dense (the dense-block kernels of the SpMM
 * stages; also contained in class 0).  Synchronises. */
int mggcn_get_profile(mggcn_model m, double* ms /*[8]*/, int64_t* launches /*[8]*/, int32_t reset);
/* Per-stage timeline (MGGCN_F_TIMELINE; the paper's Fig. 6 / Fig. 8 stage
 * timelines).  Copies up to `cap` records made
 * since the last reset, in issue order: meta[5*i ..] = {op class (as in
 * mggcn_get_profile), SpMM index within the epoch (-1 outside a SpMM), stage
 * (-1 = local stage; k >= 0 = k-th remote block / broadcast), local rank
 * index, stream (0 compute, 1 comm)}, t_ms[2*i ..] = {start, end} in device
 * milliseconds relative to the first record's start.  *count = number of
 * records available (may exceed cap).  Synchronises both streams.
 * EINVAL: cap < 0, or cap > 0 with a NULL array. */
int mggcn_get_timeline(mggcn_model m, int64_t cap, int32_t* meta, double* t_ms, int64_t* count, int32_t reset);
/* Turns MGGCN_F_TIMELINE on (on != 0) or off for the calls that follow (the
 * records cost two events per op, so timed loops run without it).  ESTATE
 * during an epoch capture. */
int mggcn_timeline_enable(mggcn_model m, int32_t on);
/* Algorithmic work of one epoch of this model's rows for the roofline
 * (DESIGN.md §6): spmm_bytes = compulsory SpMM bytes
 * (indices + rowptr + each input row once + each output row once, summed over
 * the epoch's SpMM launches), spmm_gather_bytes = cacheless gather model
 * (nnz * width * 4 B), gemm_flops, bcast_bytes = bytes received by
 * broadcasts.  Any pointer may be NULL. */
int mggcn_epoch_work(mggcn_model m, double* spmm_bytes, double* spmm_gather_bytes, double* gemm_flops,
                     double* bcast_bytes);

/* The same work model in more detail: writes min(n, 9) values into out and
 * returns 9 (or a negative error): [0] spmm_bytes (SURVEY §8(d) compulsory:
 * 4 B per non-zero of the partitioned tiles, +4 B if weighted, + rowptr + each
 * gathered row once + each output row once), [1] the same with the device
 * tiles' own structure (duplicates coalesced; index + multiplicity value per
 * entry), [2] gather bytes of the coalesced tiles (nnz * width * 4), [3] gather
 * bytes of the raw tiles, [4] gemm_flops, [5] gemm compulsory bytes
 * (4(MK + KN + MN) per product, + MN for the B3 ReLU' mask), [6] bcast_bytes
 * (received), [7] softmax-CE bytes (2 n C 4), [8] SpMM stage launches per epoch.
 * EINVAL: NULL out, n < 0. */
int mggcn_epoch_work_detail(mggcn_model m, double* out, int32_t n);

/* The remote-stage schedule the model chose (DESIGN §7 "Stage groups"): returns the
 * number of stage groups (0 = one launch per stage, the paper's BC1/BC2 schedule) and
 * writes up to cap group sizes (remote blocks per launch, in consumption order). */
int mggcn_stage_groups(mggcn_model m, int32_t* sizes, int32_t cap);

/* Dense blocks of the stage tiles (DESIGN §6 "Dense blocks"): writes min(n, 5)
 * values into out and returns 5: [0] dense 128 x 32 blocks, [1] coalesced
 * entries they cover (run on the tensor cores), [2] row groups, [3] column
 * chunks, [4] coalesced entries of every launched tile (blocks + residual CSR),
 * summed over this model's ranks and both directions (F and B tiles; one set
 * when they are shared).  The density threshold is MGGCN_DENSE_THR at
 * mggcn_model_create (default 0.04; 0 = no blocks).  EINVAL: NULL out. */
int mggcn_dense_stats(mggcn_model m, int64_t* out, int32_t n);

/* Number of kernels this library has launched in this process (all models,
 * all debug hooks).  Read before and after a timed region to count them. */
int64_t mggcn_kernel_launch_count(void);

void mggcn_graph_free(mggcn_graph g);
void mggcn_part_free(mggcn_part part);
void mggcn_model_free(mggcn_model m);

/* ------------------------------------------------- kernel-level test hooks
 * These run single ops of the hot path through the same kernels, for the
 * parity tests at full size.  They may allocate device scratch.
 * mggcn_debug_spmm: out = Â'^T B (dir 0) or Â' B (dir 1) for the model's
 *   rows, B = the model's n_local... all n rows of the permuted operand in
 *   loopback mode / P = 1 (device, ld = ldb), through the staged pipeline.
 *   In the SOLO timing mode (one rank of a P-way partition, no broadcasts) B is
 *   the rank's own block and the remote stages read the never-filled (zero) BC
 *   slots, so out = the rank's LOCAL tile times B, row-scaled on the last stage.
 * mggcn_debug_gemm: op 0: C = A·B (A MxK, B KxN); op 1: C = A·B^T (B NxK);
 *   op 2: C = A^T·B (A KxM, B KxN).  Device pointers, tcgen05 path. */
int mggcn_debug_spmm(mggcn_model m, int32_t dir, const float* B, int64_t ldb, int32_t width, float* out,
                     int64_t ldo);
int mggcn_debug_gemm(int32_t op, int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, const float* B,
                     int64_t ldb, float* C, int64_t ldc, uint32_t flags, uintptr_t stream);
/* mggcn_debug_layer: copies the layer-l activation buffer AHWB_l (this
 * model's rows, all n in loopback; d_{l+1} columns) into dst (host or device,
 * row stride ld >= d_{l+1}); synchronises.  Contents (Eq. 17-21):
 * after mggcn_forward, H_{l+1} = ReLU(Z_l) for l < L-1 and the softmax-CE
 * gradient for l = L-1; after mggcn_backward, for l < L-1, Z_{G,l} = dLoss/dZ_l
 * (Eq. 8 / 21), pre-scaled row-wise by inv_deg when layer l is GeMM-first (its
 * backward SpMM then runs on the pattern, reading C20).  EINVAL: bad layer/ld. */
int mggcn_debug_layer(mggcn_model m, int32_t layer, float* dst, int64_t ld);
/* mggcn_debug_comm_delay: delay injection for the stage/overlap rule.
 * With max_us > 0, every later broadcast (all backends) and every SpMM stage is
 * preceded by a spin kernel of a pseudo-random 0..max_us microseconds on the
 * comm or the compute stream (splitmix64 of seed and a counter), so the two
 * streams interleave differently from run to run; results must not change.
 * max_us = 0 turns it off.  EINVAL: max_us outside [0, 10000]. */
int mggcn_debug_comm_delay(mggcn_model m, uint64_t seed, int32_t max_us);
/* mggcn_debug_poison: poison-buffer injection.  With on != 0 the
 * comm stream fills every BC slot with NaN bytes right before the broadcast,
 * copy or pull into it, so a SpMM stage that read a slot outside the P:939-941
 * event rule yields NaN rows instead of silently reusing stale data.  Results
 * of a correct schedule do not change.  on = 2 is the negative control: it
 * also drops the compute stream's wait for each broadcast (and the compute-side
 * delay spins), so stages race the delayed exchange and the poison must show up
 * (tests prove the check has teeth).
 * Test hook.  EINVAL: on outside [0, 2]. */
int mggcn_debug_poison(mggcn_model m, int32_t on);

#ifdef __cplusplus
}
#endif
#endif /* MGGCN_H */
