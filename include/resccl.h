/*
 * resccl.h — C ABI of the B200-native ResCCL hot path.
 *
 * ResCCL (Liu et al., SIGCOMM '25; PAPER.md line numbers cited as P:Lx-y) executes
 * a collective-communication algorithm at primitive level: chunked send / recv /
 * recvReduceCopy / recvReduceSend / recvCopySend steps that a host-side global
 * scheduler (HPDS, Alg. 1) places on as few thread blocks as
 * possible (state-based TB allocation, Eq. 7), run by lightweight
 * generated kernels (§4.5).  Collective names: P:L436-438.
 *
 * Conventions (NCCL-like, implied by the paper's "relink and rebuild"
 * integration):
 *  - All pointers are plain device pointers (buffers) or host pointers (text,
 *    handles, info).  No torch / C++ types cross this boundary.
 *  - Counts are in elements.  AllGather's sendcount and ReduceScatter's recvcount
 *    are per rank.  count == 0 is a successful no-op.
 *  - In-place: AllReduce sendbuf == recvbuf; AllGather sendbuf == recvbuf +
 *    rank*sendcount*size; ReduceScatter recvbuf == sendbuf + rank*recvcount*size.
 *  - Collective calls only enqueue work on `stream` (cudaStream_t passed as void*;
 *    NULL = legacy default stream); they never synchronise the device.  They may be
 *    captured into CUDA graphs: the generated kernels read their flag epochs from device
 *    memory and advance them themselves (header option devepoch=1, the default), so graph
 *    replays and eager calls of the same algorithm interleave freely.  devepoch=0 and
 *    nvls=1 keep host-side epochs and refuse capture (InvalidUsage); load the algorithm
 *    before capturing (loading allocates).
 *  - Host buffers: a collective's sendbuf and/or recvbuf may be host memory (pinned
 *    for asynchronous copies; pageable works at pageable-copy speed).  The library
 *    stages it through device memory the communicator owns (grown on demand, freed
 *    by rescclCommDestroy): uploads on an internal copy stream, the collective on
 *    `stream`, downloads on a second copy stream, and `stream` waits for the last
 *    download, so the result is in recvbuf once `stream` completes.  A call is cut
 *    into pieces of RESCCL_HOST_PIECE bytes per rank (default 32 MiB) whose upload,
 *    collective and download overlap; each piece is a collective of its own over the
 *    piece's columns (its own chunk layout, so fp sums may round differently from one
 *    unpieced call).  An AllGather with a device recvbuf or a ReduceScatter with a
 *    device sendbuf runs as one piece.  The host in-place rules are the device ones.
 *    Host-buffer calls refuse CUDA-graph capture (InvalidUsage).  Staged calls of a
 *    direct=1 algorithm across processes run its staged twin (the stage is not a
 *    registered window).  The piece size is read once when a communicator is created;
 *    multi-process ranks must agree on it (rescclCommConnect: InvalidUsage otherwise).
 *    Every rank of a call must use the same placement (all host or all device buffers,
 *    per send / receive side): the placement decides the piece schedule and transport,
 *    i.e. the launches every rank must issue alike; mixed placement across processes is
 *    undefined (it hangs until the watchdog fires).  Single-process multi-device
 *    communicators refuse pageable host buffers (InvalidArgument: one host thread drives
 *    every rank, and a pageable download would block it on ranks not yet issued).  A
 *    pointer the runtime cannot classify is InvalidArgument.
 *  - ReduceScatter uses communicator-owned scratch that grows with the largest call;
 *    growing inside a CUDA-graph capture is refused (InvalidUsage): run one call of the
 *    largest size eagerly first.
 *  - All ranks issue the same collectives in the same order with the same count,
 *    dtype and op; a communicator is not thread-safe.
 *  - Every function returns a rescclResult_t; no exception crosses the ABI and the
 *    library never aborts.  rescclGetLastError() returns a message for the last
 *    failure on the calling thread.
 *  - Ownership: the caller owns buffers and streams; a communicator owns its FIFO
 *    arena, IPC mappings, compiled kernels and plans.  rescclLoadAlgorithm copies
 *    the IR text; the rescclAlgo_t lives until rescclCommDestroy.
 *
 * Execution modes:
 *  - Multi-process, one GPU per process (the production mode):
 *    rescclCommCreate -> rescclCommGetHandle -> exchange the blobs (e.g. with
 *    torch.distributed) -> rescclCommConnect; or rescclCommInit with an
 *    allgather callback.  FIFOs are CUDA-IPC-mapped peer memory over NVLink.
 *  - Single process (rescclCommInitAll): distinct devices use peer access; a
 *    device listed several times hosts several "virtual ranks" whose buffers and
 *    FIFOs share that GPU's HBM.  Virtual ranks of one device run as ONE kernel:
 *    a collective is launched when the last virtual rank of the group has issued
 *    it (on that caller's stream, ordered after the other callers' streams).
 */
#ifndef RESCCL_H_
#define RESCCL_H_

#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

#define RESCCL_VERSION 1000

typedef struct rescclComm* rescclComm_t; /* opaque; owned by the library */
typedef struct rescclAlgo* rescclAlgo_t; /* opaque; owned by its communicator */

typedef enum {
  rescclSuccess = 0,
  rescclInvalidArgument = 1, /* null pointer, bad dtype/op/count, unsupported combination */
  rescclInvalidUsage = 2,    /* IR rejected (malformed, conflicting, nranks mismatch, deadlocking
                                plan), call order violated, arena exhausted */
  rescclCudaError = 3,       /* CUDA runtime/driver or NVRTC failure */
  rescclSystemError = 4,     /* IPC / OS failure */
  rescclInternalError = 5,
  rescclTimeout = 6          /* device watchdog fired (surfaced by rescclCommGetAsyncError) */
} rescclResult_t;

typedef enum { rescclInt32 = 0, rescclFloat32 = 1, rescclFloat16 = 2, rescclBfloat16 = 3 } rescclDataType_t;

/* Sum is the paper's operator (AllReduce = ReduceScatter + AllGather);
 * max/min are order-free extras. */
typedef enum { rescclSum = 0, rescclMax = 1, rescclMin = 2 } rescclRedOp_t;

typedef enum { rescclCollAllGather = 0, rescclCollReduceScatter = 1, rescclCollAllReduce = 2 } rescclColl_t;

const char* rescclGetErrorString(rescclResult_t r);
/* Message of the last failing call on this thread (static storage, never NULL). */
const char* rescclGetLastError(void);
int rescclGetVersion(void);

/* ------------------------------------------------------------------ bootstrap */

/* Create rank `rank` of an `nranks` communicator on device `cudaDev` (multi-process
 * mode).  Allocates this rank's FIFO arena (RESCCL_ARENA_BYTES, default 128 MiB)
 * in device memory.  Not usable until rescclCommConnect. */
rescclResult_t rescclCommCreate(int rank, int nranks, int cudaDev, rescclComm_t* out);

/* Write this rank's connection blob (CUDA IPC handle of the arena plus identity)
 * into `buf`.  If buf is NULL, *len receives the required size; otherwise *len is
 * the capacity on input and the written size on output. */
rescclResult_t rescclCommGetHandle(rescclComm_t comm, void* buf, size_t* len);

/* Map every peer's arena.  handles[k] / lens[k] is rank k's blob (as written by
 * rescclCommGetHandle on rank k); handles[rank] is ignored. */
rescclResult_t rescclCommConnect(rescclComm_t comm, const void* const* handles, const size_t* lens);

/* Create + exchange + connect in one call.  `allgather` must gather `len` bytes
 * from every rank into `out` (rank-major) and return 0 on success. */
rescclResult_t rescclCommInit(rescclComm_t* out, int rank, int nranks, int cudaDev,
                              int (*allgather)(const void* in, void* out, size_t len, void* ctx), void* ctx);

/* Symmetric windows for the direct transport across processes (reading R23):
 * rescclCommRegister exports `bytes` of device memory at `ptr` (any pointer into a
 * cudaMalloc'ed / caching-allocator block; the whole block is IPC-shared) as a blob
 * (size protocol as rescclCommGetHandle); after the blobs are exchanged,
 * rescclCommRegisterConnect maps every peer's window (blobs[k] = rank k's blob) and
 * returns its id.  Every rank registers its corresponding buffer in the same order
 * with the same size.  An algorithm loaded with direct=1 then runs its direct kernel
 * when a call's send and receive buffers lie in registered windows at the same
 * offsets on every rank, and its staged twin otherwise (and for ReduceScatter). */
rescclResult_t rescclCommRegister(rescclComm_t comm, void* ptr, size_t bytes, void* blob, size_t* len);
rescclResult_t rescclCommRegisterConnect(rescclComm_t comm, const void* const* blobs, const size_t* lens,
                                         int* window);

/* Single-process communicators: comms[k] is rank k on device devlist[k].  Repeated
 * devices host virtual ranks (see "Execution modes").  devlist == NULL means all
 * ranks on device 0. */
rescclResult_t rescclCommInitAll(rescclComm_t* comms, int ndev, const int* devlist);

rescclResult_t rescclCommDestroy(rescclComm_t comm);
rescclResult_t rescclCommRank(rescclComm_t comm, int* rank);
rescclResult_t rescclCommCount(rescclComm_t comm, int* nranks);
/* CUDA device of this rank (virtual ranks: the shared device).  InvalidArgument on NULL. */
rescclResult_t rescclCommCuDevice(rescclComm_t comm, int* device);

/* Device-side failures (watchdog timeout) recorded since the last call: *err is
 * rescclSuccess or rescclTimeout.  Reads host-mapped memory; never blocks. */
rescclResult_t rescclCommGetAsyncError(rescclComm_t comm, rescclResult_t* err);

/* ------------------------------------------------------------------ algorithms */

/* Parse, analyse, schedule and lower an algorithm (Parsing ->
 * Analysis (DAG) -> Scheduling (HPDS) -> Lowering) and compile its kernel with NVRTC
 * for sm_100a on first use.  irText (copied) is the one-transfer-per-line IR:
 *     algo name=<s> coll=<allgather|reducescatter|allreduce> nranks=<N> nchunks=<N>
 *          [nwarps=16] [instances=1] [chunkbytes=1048576] [fifodepth=4]
 *          [linkmodel=pair|port] [fuse=1] [tbbudget=B]
 *     tbbudget=B (TBs = CTAs per rank): instances = floor(B / T_min) under the
 *     pair link model, or the port model (one duplex CTA per rank) with B instances when
 *     B < T_min or when linkmodel=port is given explicitly.
 *     nwarps=2 (one warp per lane) always takes the register path: the TMA lane engine
 *     needs combine warps beside each lane's leader warp.
 *     Transport and engine options: direct=0|1 (staged FIFO vs direct
 *     push / pull, R23), pushreduce=1 (with direct: rrc operands pushed into the
 *     receiver's FIFO, R31), sched=hpds|rr, tma=0|1, tmatile=B, tmastages=S, tmamin=B,
 *     bulkred=-1|0|1, lookahead=0|1|2 (R30), relaybypass=0|1 (R29), devepoch=0|1,
 *     splitfence=0|1 (one-sided release / acquire fences),
 *     postgroup=0|1 (consecutive dependency-free pull-sends posted as one group),
 *     earlyexit=0|1 (the lane engine leaves its loop right after a primitive's last post),
 *     trace=1 (TB utilisation), phase=1 (rescclGetPhaseTrace), nvls=1 (f3).
 *     t <src> <dst> <step> <chunk> <recv|rrc>
 * Environment overrides: RESCCL_INSTANCES, RESCCL_CHUNK_BYTES, RESCCL_FIFO_DEPTH,
 * RESCCL_NWARPS, RESCCL_LINK_MODEL, RESCCL_FUSE, RESCCL_TB_BUDGET.
 * The loaded algorithm becomes the active one for its collective; with none
 * loaded, the built-in ring is used.  Size-based selection: header options
 * [minbytes=a] [maxbytes=b] give the range of per-rank buffer sizes S (AllReduce
 * count x elt; AllGather / ReduceScatter N x count x elt) an algorithm serves; a call
 * runs the most recently loaded or activated algorithm of its collective whose range
 * holds its S (default range: every size), so e.g. a full-mesh schedule can serve small
 * messages and a ring large ones.  All ranks must load the same algorithms in the same
 * order.  InvalidUsage: nranks != communicator size, invalid IR (I6), same-step
 * conflicts, deadlocking plan. */
rescclResult_t rescclLoadAlgorithm(rescclComm_t comm, const char* irText, rescclAlgo_t* out);

/* Make a previously loaded algorithm the active one for its collective (and the most
 * recent one for size-based selection). */
rescclResult_t rescclSetActiveAlgorithm(rescclComm_t comm, rescclAlgo_t algo);

/* JSON description of the lowered plan (Pr, per-rank CTAs/lanes/primitives,
 * connection groups, TB counts, layout).  Same size protocol as rescclCommGetHandle. */
rescclResult_t rescclGetPlanInfo(rescclAlgo_t algo, char* json, size_t* len);

/* TB utilisation of the last launch of `algo` (§5.4): per lane
 * ("TB" in the paper's count) its lifetime and the time it spent busy-waiting on
 * dependencies, payload or credit; plus Comm Time = 1 - mean idle ratio, Avg Idle,
 * Max Idle (Table 3's columns).  Requires the algorithm loaded with trace=1 (or
 * RESCCL_TRACE=1) and the launch finished (synchronise the stream first). */
rescclResult_t rescclGetTbUtilization(rescclAlgo_t algo, char* json, size_t* len);

/* Phase records of the last launch of `algo` (where a hop's time
 * goes).  Requires the algorithm loaded with phase=1.  Every lane leader writes one
 * record per (primitive, micro-batch) into device memory with %globaltimer stamps;
 * this call synchronises the device and copies them out as u64 words:
 *   [0] blocks, [1] first global block, [2] records per (block, lane) P, [3] instances,
 *   then for block b (launch-relative) and lane l (0 send, 1 recv) P records of 8 words
 *   at 4 + (2b + l)·8P.  Record 0 = lane header {entry ns, exit ns, records, rank, cta,
 *   instance}; record k >= 1 = {prim << 32 | mb << 8 | kind, t0, t1, t2, t3, t4},
 *   kind 0 register path (t0 start, t1 dependencies met, t2 flag / credit met, t3 data
 *   moved, t4 posted), 1 flag-only primitive (t0 start of wait, t1 dependencies met /
 *   readable or writable posted, t2 peer's payload seen, t4 posted), 2 TMA engine
 *   (t0 previous post, t1 ready, t3 stores complete, t4 posted); 0 = not recorded.
 * buf NULL: *len = bytes needed.  Ownership: the caller owns buf.  InvalidUsage when the
 * algorithm was not loaded with phase=1 or has not run; CudaError on copy failure. */
rescclResult_t rescclGetPhaseTrace(rescclAlgo_t algo, void* buf, size_t* len);

/* ------------------------------------------------------------------ collectives */

/* out_r[i] = sum_k in_k[i].  sendbuf/recvbuf: count elements each. */
rescclResult_t rescclAllReduce(const void* sendbuf, void* recvbuf, size_t count, rescclDataType_t dtype,
                               rescclRedOp_t op, rescclComm_t comm, void* stream);
/* out_r[k*sendcount + i] = in_k[i].  recvbuf: nranks*sendcount elements. */
rescclResult_t rescclAllGather(const void* sendbuf, void* recvbuf, size_t sendcount, rescclDataType_t dtype,
                               rescclComm_t comm, void* stream);
/* out_r[i] = sum_k in_k[r*recvcount + i].  sendbuf: nranks*recvcount elements. */
rescclResult_t rescclReduceScatter(const void* sendbuf, void* recvbuf, size_t recvcount,
                                   rescclDataType_t dtype, rescclRedOp_t op, rescclComm_t comm, void* stream);

/* ------------------------------------------------------------------ f3: NVLS (NVLink SHARP) windows */

/* not in the paper: the NVSwitch-SHARP transport variant.  An NVLS
 * window is `bytes` of device memory on every rank, all bound into one multicast object,
 * so that multimem.ld_reduce through the multicast alias returns the switch-computed
 * reduction of every rank's copy and multimem.st lands in every rank's copy.  An
 * algorithm loaded with the header option nvls=1 (env RESCCL_NVLS=1; CTAs per rank:
 * nvlsctas=16) runs a call on the NVLS kernel when
 *   - its send and receive buffers lie in NVLS windows at 4-byte-aligned offsets, the
 *     same on every rank (allocate windows in the same order and size everywhere),
 *   - each rank's block (AR: the buffer; RS: recvcount; AG: sendcount) is a whole number
 *     of 4-byte granules (2-byte dtypes: even counts), and
 *   - the op has a multimem form (all but float32 max/min);
 * otherwise the algorithm's primitive plan runs.  The NVLS schedule on the collective's
 * chunk layout: ReduceScatter mred(r): <r,r> := (+)_k <k,r>; AllGather mcast(r):
 * <k,r> := <r,r> for all k; AllReduce = mred + mcast of 16-byte-aligned slices
 * (reading R28).  bf16/fp16 sums accumulate in fp32 inside the switch.
 * Windows are owned by the communicator (freed by rescclNvlsFree or rescclCommDestroy);
 * the returned pointer is the window's first byte (4 KiB aligned).
 * CudaError when the driver or the fabric refuses multicast (message names the call and
 * the failing rank); every rank of a multi-process allocation returns it. */

/* *supported = CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED of the communicator's device
 * (0 for virtual ranks, which share one device). */
rescclResult_t rescclNvlsSupported(rescclComm_t comm, int* supported);
/* Multi-process, collective over all ranks: rank 0 creates the multicast object and
 * exports a fabric handle, the `allgather` callback (as for rescclCommInit) carries it
 * and two status rounds; every rank makes the same three callback calls even when a
 * step fails locally, so a failure anywhere returns an error everywhere. */
rescclResult_t rescclNvlsAlloc(rescclComm_t comm, size_t bytes, int (*allgather)(const void* in, void* out, size_t len, void* ctx),
                               void* ctx, void** ptr);
/* Single process, one device per rank (rescclCommInitAll with distinct devices):
 * comms[k] is rank k of n; ptrs[k] receives rank k's window. */
rescclResult_t rescclNvlsAllocAll(rescclComm_t* comms, int n, size_t bytes, void** ptrs);
rescclResult_t rescclNvlsFree(rescclComm_t comm, void* ptr);

/* ------------------------------------------------------------------ host-only tools (no GPU needed) */

/* Built-in generators (name in ring|dbt|hm|synth; opts "g=4 seed=0 fanout=2").
 * Writes IR text; size protocol as above. */
rescclResult_t rescclGenerateIr(const char* name, rescclColl_t coll, int nranks, const char* opts, char* text,
                                size_t* len);
/* ResCCLang front end (BNF Fig. 14): execute a `def ResCCLAlgo(...):`
 * program -- e.g. the paper's Fig. 16 listing -- and write the resulting IR text.
 * rescclLoadAlgorithm / rescclPlanIr also accept such programs directly.
 * InvalidUsage on syntax errors (message names the line). */
rescclResult_t rescclParseResCCLang(const char* program, char* irText, size_t* len);
/* Workflow phase timings (Fig. 10a): Parsing, Analysis (DAG),
 * Scheduling (HPDS / RR), Lowering (translation, TB allocation, rank-0 kernel source)
 * and, if `verify`, the blocking-model deadlock check; JSON with counts and ms. */
rescclResult_t rescclProfilePlanner(const char* program, const char* opts, int verify, char* json, size_t* len);
/* Plan an IR (header keys as for rescclLoadAlgorithm; `opts` overrides them) and
 * write the plan JSON. */
rescclResult_t rescclPlanIr(const char* irText, const char* opts, char* json, size_t* len);
/* Generated CUDA source of an IR's kernel for ranks [rank_lo, rank_hi). */
rescclResult_t rescclCodegenIr(const char* irText, const char* opts, int rank_lo, int rank_hi, char* src,
                               size_t* len);
/* NVRTC-compile the kernel of an IR for sm_100a (no GPU needed); *cubin_bytes
 * receives the cubin size. */
rescclResult_t rescclCompileIr(const char* irText, const char* opts, rescclDataType_t dtype, rescclRedOp_t op,
                               size_t* cubin_bytes);
/* NVRTC-compile the NVLS kernel of a collective for sm_100a (no GPU needed); InvalidArgument
 * for a bad coll/dtype/op.  (float32 max/min compile but are never launched.) */
rescclResult_t rescclCompileNvls(rescclColl_t coll, rescclDataType_t dtype, rescclRedOp_t op, size_t* cubin_bytes);
/* Control-only blocking simulation of a planned IR (invariant I4): *ok = 1 if the
 * plan completes for FIFO depth K and n_mb micro-batches. */
rescclResult_t rescclCheckDeadlock(const char* irText, const char* opts, int K, int n_mb, int* ok);
/* Wall-clock timeline of a planned IR under the alpha-beta model with link contention
 * (Eq. 1; task-level execution, Eq. 5; reading R27), and the
 * state-based merge of Eq. 7 evaluated on wall-clock activity active_l(t)
 * (P:L1852-1885).  `params`: "count=<elements per rank buffer> elt=<2|4> alpha=<s>
 * beta=<s/byte> gamma=<s>"; the micro-batch geometry follows the plan's chunkbytes
 * and instances (`opts` / IR header), K = fifodepth.  Writes JSON: makespan_s,
 * comm_time / avg_idle / max_idle over lanes (Table 3's metrics, predicted), the
 * largest contention z, and per rank the connections' activity intervals and the
 * merged lane counts (wall clock vs pipeline index).  InvalidUsage if the plan
 * deadlocks. */
rescclResult_t rescclSimulateTimeline(const char* irText, const char* opts, const char* params, char* json,
                                      size_t* len);

#ifdef __cplusplus
}
#endif
#endif /* RESCCL_H_ */
