/*
 * resccl_nccl.h — NCCL-symbol shim over the ResCCL C ABI (libresccl_nccl.so).
 *
 * The paper integrates ResCCL into Megatron-LM by "relink and rebuild" (PAPER.md
 * P:L2624-2628): the framework keeps calling the NCCL API and is linked against ResCCL
 * instead.  This header declares the NCCL subset the shim exports, with NCCL's names,
 * enum values and argument order, so an application built against nccl.h links against
 * libresccl_nccl.so unchanged (or preloads it).  Every call forwards to include/resccl.h:
 *
 *   ncclAllReduce     -> rescclAllReduce      (ncclSum / ncclMax / ncclMin)
 *   ncclAllGather     -> rescclAllGather
 *   ncclReduceScatter -> rescclReduceScatter  (ncclSum / ncclMax / ncclMin)
 *   ncclBroadcast     -> rescclAllReduce of the root's bits with zeros from every other
 *                        rank (on an int32 view when the byte count is a multiple of 4:
 *                        bit-exact; otherwise in the element type, where x + 0 = x
 *                        except -0.0 -> +0.0)
 *
 * Datatypes: ncclInt32, ncclFloat32, ncclFloat16, ncclBfloat16 (and any type for
 * ncclBroadcast whose byte count is a multiple of 4).  Other types and ncclProd /
 * ncclAvg return ncclInvalidArgument.  ncclGroupStart / ncclGroupEnd are accepted and
 * do nothing: every call is enqueued on its stream as it is made, so a group of calls
 * from one thread on one communicator works; grouping several communicators of one
 * thread (one thread driving several GPUs) is not supported -- use ncclCommInitAll.
 *
 * Bootstrap (ncclGetUniqueId / ncclCommInitRank): the id carries a TCP rendezvous
 * address (RESCCL_SHIM_ADDR, default 127.0.0.1 -- one box) served by a
 * thread of the process that called ncclGetUniqueId; every rank sends its connection
 * blob (rescclCommGetHandle) and receives all of them back (rescclCommConnect).  The id
 * is valid for one communicator.  Errors: ncclSystemError on socket failures or a
 * rendezvous timeout (RESCCL_SHIM_TIMEOUT_S, default 300 s); ncclInvalidUsage /
 * ncclUnhandledCudaError mirror rescclInvalidUsage / rescclCudaError.  The device is
 * the caller's current CUDA device (NCCL's rule).  Ownership: as in NCCL; a
 * communicator is released by ncclCommDestroy.
 */
#ifndef RESCCL_NCCL_H_
#define RESCCL_NCCL_H_

#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

#define NCCL_UNIQUE_ID_BYTES 128
typedef struct { char internal[NCCL_UNIQUE_ID_BYTES]; } ncclUniqueId;
typedef struct ncclComm* ncclComm_t;

typedef enum {
  ncclSuccess = 0,
  ncclUnhandledCudaError = 1,
  ncclSystemError = 2,
  ncclInternalError = 3,
  ncclInvalidArgument = 4,
  ncclInvalidUsage = 5,
  ncclRemoteError = 6,
  ncclInProgress = 7
} ncclResult_t;

typedef enum {
  ncclInt8 = 0, ncclChar = 0, ncclUint8 = 1, ncclInt32 = 2, ncclInt = 2, ncclUint32 = 3,
  ncclInt64 = 4, ncclUint64 = 5, ncclFloat16 = 6, ncclHalf = 6, ncclFloat32 = 7, ncclFloat = 7,
  ncclFloat64 = 8, ncclDouble = 8, ncclBfloat16 = 9
} ncclDataType_t;

typedef enum { ncclSum = 0, ncclProd = 1, ncclMax = 2, ncclMin = 3, ncclAvg = 4 } ncclRedOp_t;

ncclResult_t ncclGetVersion(int* version);
ncclResult_t ncclGetUniqueId(ncclUniqueId* uniqueId);
ncclResult_t ncclCommInitRank(ncclComm_t* comm, int nranks, ncclUniqueId commId, int rank);
ncclResult_t ncclCommInitAll(ncclComm_t* comms, int ndev, const int* devlist);
ncclResult_t ncclCommDestroy(ncclComm_t comm);
ncclResult_t ncclCommAbort(ncclComm_t comm);
ncclResult_t ncclCommCount(const ncclComm_t comm, int* count);
ncclResult_t ncclCommCuDevice(const ncclComm_t comm, int* device);
ncclResult_t ncclCommUserRank(const ncclComm_t comm, int* rank);
ncclResult_t ncclCommGetAsyncError(ncclComm_t comm, ncclResult_t* asyncError);
const char* ncclGetErrorString(ncclResult_t result);
const char* ncclGetLastError(ncclComm_t comm);
ncclResult_t ncclGroupStart(void);
ncclResult_t ncclGroupEnd(void);
/* stream: cudaStream_t */
ncclResult_t ncclAllReduce(const void* sendbuff, void* recvbuff, size_t count, ncclDataType_t datatype,
                           ncclRedOp_t op, ncclComm_t comm, void* stream);
ncclResult_t ncclAllGather(const void* sendbuff, void* recvbuff, size_t sendcount, ncclDataType_t datatype,
                           ncclComm_t comm, void* stream);
ncclResult_t ncclReduceScatter(const void* sendbuff, void* recvbuff, size_t recvcount, ncclDataType_t datatype,
                               ncclRedOp_t op, ncclComm_t comm, void* stream);
ncclResult_t ncclBroadcast(const void* sendbuff, void* recvbuff, size_t count, ncclDataType_t datatype, int root,
                           ncclComm_t comm, void* stream);

/* Test hook (not NCCL API): the rendezvous alone -- rank `rank` of `nranks` sends `blob`
 * to the id's server and receives every rank's blob, concatenated in rank order into
 * `out` with their lengths in `lens`.  Lets the host-side bootstrap be tested without a
 * GPU.  *out_len: capacity in, bytes written out. */
ncclResult_t rescclShimExchange(const ncclUniqueId* id, int rank, int nranks, const void* blob, size_t len,
                                void* out, size_t* out_len, size_t* lens);

#ifdef __cplusplus
}
#endif
#endif /* RESCCL_NCCL_H_ */
