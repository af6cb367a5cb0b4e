// NCCL-symbol shim over the ResCCL C ABI (include/resccl_nccl.h): the "relink and
// rebuild" integration of PAPER.md P:L2624-2628.  Argument mapping only; every
// collective runs in libresccl.so's generated kernels.
#include "resccl_nccl.h"

#include <arpa/inet.h>
#include <dlfcn.h>
#include <netinet/in.h>
#include <netinet/tcp.h>
#include <poll.h>
#include <sys/socket.h>
#include <unistd.h>

#include <chrono>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <random>
#include <string>
#include <thread>
#include <vector>

#include "resccl.h"

namespace {

thread_local std::string g_err;

ncclResult_t from_resccl(rescclResult_t r) {
  switch (r) {
    case rescclSuccess: return ncclSuccess;
    case rescclInvalidArgument: return ncclInvalidArgument;
    case rescclInvalidUsage: return ncclInvalidUsage;
    case rescclCudaError: return ncclUnhandledCudaError;
    case rescclSystemError: return ncclSystemError;
    case rescclTimeout: return ncclRemoteError;
    default: return ncclInternalError;
  }
}

ncclResult_t fwd(rescclResult_t r) {
  if (r != rescclSuccess) g_err = rescclGetLastError();
  return from_resccl(r);
}

ncclResult_t fail(ncclResult_t r, const std::string& m) {
  g_err = m;
  return r;
}

bool dtype_of(ncclDataType_t t, rescclDataType_t* out) {
  switch (t) {
    case ncclInt32: *out = rescclInt32; return true;
    case ncclFloat32: *out = rescclFloat32; return true;
    case ncclFloat16: *out = rescclFloat16; return true;
    case ncclBfloat16: *out = rescclBfloat16; return true;
    default: return false;
  }
}
size_t dtype_bytes(ncclDataType_t t) {
  switch (t) {
    case ncclInt8: case ncclUint8: return 1;
    case ncclFloat16: case ncclBfloat16: return 2;
    case ncclInt32: case ncclUint32: case ncclFloat32: return 4;
    default: return 8;
  }
}
bool op_of(ncclRedOp_t o, rescclRedOp_t* out) {
  switch (o) {
    case ncclSum: *out = rescclSum; return true;
    case ncclMax: *out = rescclMax; return true;
    case ncclMin: *out = rescclMin; return true;
    default: return false;
  }
}

// ---- the few driver entry points the shim needs (no cudart link: libresccl.so owns it)
struct Drv {
  int (*CtxGetDevice)(int*) = nullptr;
  int (*MemsetD32Async)(unsigned long long, unsigned int, size_t, void*) = nullptr;
  int (*MemsetD8Async)(unsigned long long, unsigned char, size_t, void*) = nullptr;
  bool ok = false;
};
Drv& drv() {
  static Drv d = [] {
    Drv x;
    void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return x;
    x.CtxGetDevice = (int (*)(int*))dlsym(h, "cuCtxGetDevice");
    x.MemsetD32Async = (int (*)(unsigned long long, unsigned int, size_t, void*))dlsym(h, "cuMemsetD32Async");
    x.MemsetD8Async = (int (*)(unsigned long long, unsigned char, size_t, void*))dlsym(h, "cuMemsetD8Async");
    x.ok = x.CtxGetDevice && x.MemsetD32Async && x.MemsetD8Async;
    return x;
  }();
  return d;
}

// ---- rendezvous: id = magic, IPv4, port, nonce
struct IdBody {
  char magic[8];
  uint32_t addr;   // network order
  uint16_t port;   // network order
  uint16_t pad;
  uint64_t nonce;
};
static_assert(sizeof(IdBody) <= NCCL_UNIQUE_ID_BYTES, "id");

double timeout_s() {
  const char* v = getenv("RESCCL_SHIM_TIMEOUT_S");
  double t = v ? atof(v) : 300.0;
  return t > 0 ? t : 300.0;
}

bool send_all(int fd, const void* p, size_t n) {
  const char* c = (const char*)p;
  while (n) {
    ssize_t k = ::send(fd, c, n, MSG_NOSIGNAL);
    if (k <= 0) return false;
    c += k;
    n -= (size_t)k;
  }
  return true;
}
bool recv_all(int fd, void* p, size_t n) {
  char* c = (char*)p;
  while (n) {
    ssize_t k = ::recv(fd, c, n, 0);
    if (k <= 0) return false;
    c += k;
    n -= (size_t)k;
  }
  return true;
}

struct Hello {
  uint64_t nonce;
  int32_t rank, nranks;
  uint64_t len;
};

// server: collect nranks hellos, answer every client with all blobs, exit
void serve(int lfd, uint64_t nonce) {
  const auto deadline = std::chrono::steady_clock::now() + std::chrono::duration<double>(timeout_s());
  std::vector<int> fds;
  std::vector<std::string> blobs;
  std::vector<int> have;
  int nranks = -1, got = 0;
  while (nranks < 0 || got < nranks) {
    const double left = std::chrono::duration<double>(deadline - std::chrono::steady_clock::now()).count();
    if (left <= 0) break;
    pollfd p{lfd, POLLIN, 0};
    if (poll(&p, 1, (int)(left * 1000) + 1) <= 0) continue;
    int fd = accept(lfd, nullptr, nullptr);
    if (fd < 0) continue;
    Hello h;
    if (!recv_all(fd, &h, sizeof(h)) || h.nonce != nonce || h.nranks <= 0 || h.rank < 0 || h.rank >= h.nranks ||
        (nranks >= 0 && h.nranks != nranks) || h.len > (64u << 20)) {
      close(fd);
      continue;
    }
    std::string b(h.len, '\0');
    if (!recv_all(fd, &b[0], h.len)) {
      close(fd);
      continue;
    }
    if (nranks < 0) {
      nranks = h.nranks;
      blobs.assign(nranks, std::string());
      have.assign(nranks, 0);
    }
    if (have[h.rank]) {
      close(fd);
      continue;
    }
    have[h.rank] = 1;
    blobs[h.rank] = b;
    fds.push_back(fd);
    ++got;
  }
  if (nranks > 0 && got == nranks) {
    std::vector<uint64_t> lens(nranks);
    for (int r = 0; r < nranks; ++r) lens[r] = blobs[r].size();
    for (int fd : fds) {
      bool ok = send_all(fd, lens.data(), lens.size() * 8);
      for (int r = 0; ok && r < nranks; ++r) ok = send_all(fd, blobs[r].data(), blobs[r].size());
    }
  }
  for (int fd : fds) close(fd);
  close(lfd);
}

ncclResult_t exchange(const ncclUniqueId& id, int rank, int nranks, const std::string& mine,
                      std::vector<std::string>* all) {
  IdBody b;
  std::memcpy(&b, id.internal, sizeof(b));
  if (std::memcmp(b.magic, "RESCCLID", 8) != 0) return fail(ncclInvalidArgument, "not a ResCCL unique id");
  sockaddr_in sa{};
  sa.sin_family = AF_INET;
  sa.sin_addr.s_addr = b.addr;
  sa.sin_port = b.port;
  const auto deadline = std::chrono::steady_clock::now() + std::chrono::duration<double>(timeout_s());
  int fd = -1;
  while (true) {
    fd = socket(AF_INET, SOCK_STREAM, 0);
    if (fd < 0) return fail(ncclSystemError, "socket failed");
    if (connect(fd, (sockaddr*)&sa, sizeof(sa)) == 0) break;
    close(fd);
    fd = -1;
    if (std::chrono::steady_clock::now() > deadline) return fail(ncclSystemError, "rendezvous connect timed out");
    std::this_thread::sleep_for(std::chrono::milliseconds(20));
  }
  Hello h{b.nonce, rank, nranks, (uint64_t)mine.size()};
  bool ok = send_all(fd, &h, sizeof(h)) && send_all(fd, mine.data(), mine.size());
  std::vector<uint64_t> lens(nranks);
  ok = ok && recv_all(fd, lens.data(), lens.size() * 8);
  all->assign(nranks, std::string());
  for (int r = 0; ok && r < nranks; ++r) {
    if (lens[r] > (64u << 20)) ok = false;
    else {
      (*all)[r].resize(lens[r]);
      ok = recv_all(fd, &(*all)[r][0], lens[r]);
    }
  }
  close(fd);
  return ok ? ncclSuccess : fail(ncclSystemError, "rendezvous exchange failed (peer missing or timed out)");
}

}  // namespace

extern "C" {

ncclResult_t ncclGetVersion(int* version) {
  if (!version) return fail(ncclInvalidArgument, "version is NULL");
  *version = 22800;  // the NCCL API level the shim mirrors (2.28); ResCCL's own: rescclGetVersion
  return ncclSuccess;
}

const char* ncclGetErrorString(ncclResult_t r) {
  switch (r) {
    case ncclSuccess: return "no error";
    case ncclUnhandledCudaError: return "unhandled cuda error (ResCCL)";
    case ncclSystemError: return "unhandled system error (ResCCL)";
    case ncclInternalError: return "internal error (ResCCL)";
    case ncclInvalidArgument: return "invalid argument (ResCCL)";
    case ncclInvalidUsage: return "invalid usage (ResCCL)";
    case ncclRemoteError: return "remote process exited or there was a network error (ResCCL)";
    case ncclInProgress: return "operation in progress";
  }
  return "unknown result code";
}

const char* ncclGetLastError(ncclComm_t) { return g_err.c_str(); }

ncclResult_t ncclGetUniqueId(ncclUniqueId* id) {
  if (!id) return fail(ncclInvalidArgument, "uniqueId is NULL");
  const char* a = getenv("RESCCL_SHIM_ADDR");
  sockaddr_in sa{};
  sa.sin_family = AF_INET;
  if (inet_pton(AF_INET, a ? a : "127.0.0.1", &sa.sin_addr) != 1) return fail(ncclInvalidArgument, "bad RESCCL_SHIM_ADDR");
  sa.sin_port = 0;
  int lfd = socket(AF_INET, SOCK_STREAM, 0);
  if (lfd < 0) return fail(ncclSystemError, "socket failed");
  int one = 1;
  setsockopt(lfd, SOL_SOCKET, SO_REUSEADDR, &one, sizeof(one));
  socklen_t sl = sizeof(sa);
  if (bind(lfd, (sockaddr*)&sa, sizeof(sa)) != 0 || listen(lfd, 256) != 0 || getsockname(lfd, (sockaddr*)&sa, &sl) != 0) {
    close(lfd);
    return fail(ncclSystemError, "bind/listen failed");
  }
  IdBody b{};
  std::memcpy(b.magic, "RESCCLID", 8);
  b.addr = sa.sin_addr.s_addr;
  b.port = sa.sin_port;
  b.nonce = std::random_device{}() ^ ((uint64_t)std::random_device{}() << 32) ^
            (uint64_t)std::chrono::steady_clock::now().time_since_epoch().count();
  std::memset(id->internal, 0, sizeof(id->internal));
  std::memcpy(id->internal, &b, sizeof(b));
  std::thread(serve, lfd, b.nonce).detach();
  return ncclSuccess;
}

ncclResult_t rescclShimExchange(const ncclUniqueId* id, int rank, int nranks, const void* blob, size_t len,
                                void* out, size_t* out_len, size_t* lens) {
  if (!id || !out_len || !lens || (len && !blob) || nranks <= 0 || rank < 0 || rank >= nranks)
    return fail(ncclInvalidArgument, "bad argument");
  std::vector<std::string> all;
  ncclResult_t r = exchange(*id, rank, nranks, std::string((const char*)blob, len), &all);
  if (r != ncclSuccess) return r;
  size_t tot = 0;
  for (auto& s : all) tot += s.size();
  if (!out || *out_len < tot) {
    *out_len = tot;
    return fail(ncclInvalidArgument, "output buffer too small");
  }
  size_t o = 0;
  for (int q = 0; q < nranks; ++q) {
    std::memcpy((char*)out + o, all[q].data(), all[q].size());
    lens[q] = all[q].size();
    o += all[q].size();
  }
  *out_len = tot;
  return ncclSuccess;
}

ncclResult_t ncclCommInitRank(ncclComm_t* comm, int nranks, ncclUniqueId id, int rank) {
  if (!comm) return fail(ncclInvalidArgument, "comm is NULL");
  if (!drv().ok) return fail(ncclUnhandledCudaError, "libcuda.so.1 not available");
  int dev = 0;
  if (drv().CtxGetDevice(&dev) != 0) dev = 0;  // no current context yet: device 0 (NCCL: current device)
  rescclComm_t c = nullptr;
  ncclResult_t r = fwd(rescclCommCreate(rank, nranks, dev, &c));
  if (r != ncclSuccess) return r;
  size_t n = 0;
  if ((r = fwd(rescclCommGetHandle(c, nullptr, &n))) != ncclSuccess) return r;
  std::string mine(n, '\0');
  if ((r = fwd(rescclCommGetHandle(c, &mine[0], &n))) != ncclSuccess) return r;
  std::vector<std::string> all;
  if ((r = exchange(id, rank, nranks, mine, &all)) != ncclSuccess) {
    rescclCommDestroy(c);
    return r;
  }
  std::vector<const void*> ptrs(nranks);
  std::vector<size_t> lens(nranks);
  for (int q = 0; q < nranks; ++q) {
    ptrs[q] = all[q].data();
    lens[q] = all[q].size();
  }
  if ((r = fwd(rescclCommConnect(c, ptrs.data(), lens.data()))) != ncclSuccess) {
    rescclCommDestroy(c);
    return r;
  }
  *comm = (ncclComm_t)c;
  return ncclSuccess;
}

ncclResult_t ncclCommInitAll(ncclComm_t* comms, int ndev, const int* devlist) {
  if (!comms || ndev <= 0) return fail(ncclInvalidArgument, "bad argument");
  std::vector<int> d(ndev);
  for (int i = 0; i < ndev; ++i) d[i] = devlist ? devlist[i] : i;  // NCCL: devlist NULL = devices 0..ndev-1
  return fwd(rescclCommInitAll((rescclComm_t*)comms, ndev, d.data()));
}

ncclResult_t ncclCommDestroy(ncclComm_t comm) { return fwd(rescclCommDestroy((rescclComm_t)comm)); }
ncclResult_t ncclCommAbort(ncclComm_t comm) { return fwd(rescclCommDestroy((rescclComm_t)comm)); }

ncclResult_t ncclCommCount(const ncclComm_t comm, int* count) {
  return fwd(rescclCommCount((rescclComm_t)comm, count));
}
ncclResult_t ncclCommUserRank(const ncclComm_t comm, int* rank) {
  return fwd(rescclCommRank((rescclComm_t)comm, rank));
}
ncclResult_t ncclCommCuDevice(const ncclComm_t comm, int* device) {
  return fwd(rescclCommCuDevice((rescclComm_t)comm, device));
}
ncclResult_t ncclCommGetAsyncError(ncclComm_t comm, ncclResult_t* asyncError) {
  if (!asyncError) return fail(ncclInvalidArgument, "asyncError is NULL");
  rescclResult_t e = rescclSuccess;
  ncclResult_t r = fwd(rescclCommGetAsyncError((rescclComm_t)comm, &e));
  *asyncError = from_resccl(e);
  return r;
}

ncclResult_t ncclGroupStart(void) { return ncclSuccess; }
ncclResult_t ncclGroupEnd(void) { return ncclSuccess; }

ncclResult_t ncclAllReduce(const void* sendbuff, void* recvbuff, size_t count, ncclDataType_t datatype,
                           ncclRedOp_t op, ncclComm_t comm, void* stream) {
  rescclDataType_t t;
  rescclRedOp_t o;
  if (!dtype_of(datatype, &t)) return fail(ncclInvalidArgument, "datatype not supported by ResCCL");
  if (!op_of(op, &o)) return fail(ncclInvalidArgument, "reduction op not supported by ResCCL (sum/max/min)");
  return fwd(rescclAllReduce(sendbuff, recvbuff, count, t, o, (rescclComm_t)comm, stream));
}

ncclResult_t ncclAllGather(const void* sendbuff, void* recvbuff, size_t sendcount, ncclDataType_t datatype,
                           ncclComm_t comm, void* stream) {
  rescclDataType_t t;
  if (!dtype_of(datatype, &t)) return fail(ncclInvalidArgument, "datatype not supported by ResCCL");
  return fwd(rescclAllGather(sendbuff, recvbuff, sendcount, t, (rescclComm_t)comm, stream));
}

ncclResult_t ncclReduceScatter(const void* sendbuff, void* recvbuff, size_t recvcount, ncclDataType_t datatype,
                               ncclRedOp_t op, ncclComm_t comm, void* stream) {
  rescclDataType_t t;
  rescclRedOp_t o;
  if (!dtype_of(datatype, &t)) return fail(ncclInvalidArgument, "datatype not supported by ResCCL");
  if (!op_of(op, &o)) return fail(ncclInvalidArgument, "reduction op not supported by ResCCL (sum/max/min)");
  return fwd(rescclReduceScatter(sendbuff, recvbuff, recvcount, t, o, (rescclComm_t)comm, stream));
}

ncclResult_t ncclBroadcast(const void* sendbuff, void* recvbuff, size_t count, ncclDataType_t datatype, int root,
                           ncclComm_t comm, void* stream) {
  int rank = 0;
  ncclResult_t r = fwd(rescclCommRank((rescclComm_t)comm, &rank));
  if (r != ncclSuccess) return r;
  const size_t bytes = count * dtype_bytes(datatype);
  if (bytes == 0) return ncclSuccess;
  rescclDataType_t t;
  size_t n;
  if (bytes % 4 == 0) {  // bit-exact: integer sum of the root's words and zeros
    t = rescclInt32;
    n = bytes / 4;
  } else if (dtype_of(datatype, &t)) {
    n = count;
  } else {
    return fail(ncclInvalidArgument, "broadcast: byte count not a multiple of 4 for this datatype");
  }
  if (!drv().ok) return fail(ncclUnhandledCudaError, "libcuda.so.1 not available");
  const void* src = recvbuff;
  if (rank == root) {
    src = sendbuff;
  } else {
    const int e = (bytes % 4 == 0) ? drv().MemsetD32Async((unsigned long long)recvbuff, 0u, bytes / 4, stream)
                                   : drv().MemsetD8Async((unsigned long long)recvbuff, 0, bytes, stream);
    if (e != 0) return fail(ncclUnhandledCudaError, "cuMemsetAsync failed");
  }
  return fwd(rescclAllReduce(src, recvbuff, n, t, rescclSum, (rescclComm_t)comm, stream));
}

}  // extern "C"
