// ResCCL control plane + C ABI (include/resccl.h).
//
// The paper's middle layer is "CPU-side coordination and management for the runtime"
// (P:L2030-2035).  Here it owns: communicators and their FIFO arenas, CUDA-IPC
// mapping of peer arenas (NVLink peer memory), loading algorithms (parse -> DAG ->
// HPDS -> lower), NVRTC compilation of the generated kernel for
// sm_100a (cached per plan/dtype/op), per-call geometry and the launch.
#include <cuda.h>
#include <cuda_runtime.h>
#include <nvrtc.h>

#include <unistd.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <sstream>
#include <string>
#include <vector>

#include "../../../include/resccl.h"
#include "../plan/codegen.h"
#include "../plan/timeline.h"
#include "../plan/ir.h"
#include "../plan/plan.h"

static const char* kDeviceSrc =
#include "device_src.inc"
    ;

namespace {

using namespace resccl;
constexpr int kMaxR = 32;
#define RESCCL_PH_MAX_HOST 96  // = RESCCL_PH_MAX (resccl_device.cuh): phase records per (block, lane)

// host mirror of rdev::KArgs (resccl_device.cuh)
struct KArgs {
  char* arena[kMaxR];
  const char* sendbuf[kMaxR];
  char* recvbuf[kMaxR];
  char* scratch[kMaxR];
  unsigned long long mb_base;
  long long count, C, M, Mi;
  int n_mb;
  int block_base;
  int* err;
  unsigned long long timeout_ns;
  unsigned long long* trace;
  unsigned long long epoch;
  unsigned long long* epochs;  // device-side epochs {mb_base, epoch, CTAs done}, or null
  unsigned long long* phase;   // phase=1: per-(block, lane) phase records (device memory), or null
};

thread_local std::string g_last_error;

struct Error {
  rescclResult_t code;
  std::string msg;
};

[[noreturn]] void fail(rescclResult_t c, const std::string& m) { throw Error{c, m}; }

void cuda_check(cudaError_t e, const char* what) {
  if (e != cudaSuccess) fail(rescclCudaError, std::string(what) + ": " + cudaGetErrorString(e));
}

// ---------------------------------------------------------------- driver entry points (no libcuda link)
struct Driver {
  CUresult (*ModuleLoadData)(CUmodule*, const void*) = nullptr;
  CUresult (*ModuleGetFunction)(CUfunction*, CUmodule, const char*) = nullptr;
  CUresult (*ModuleUnload)(CUmodule) = nullptr;
  CUresult (*LaunchCooperativeKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                                      unsigned, CUstream, void**) = nullptr;
  CUresult (*LaunchKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                           CUstream, void**, void**) = nullptr;
  CUresult (*GetErrorString)(CUresult, const char**) = nullptr;
  CUresult (*FuncSetAttribute)(CUfunction, CUfunction_attribute, int) = nullptr;
  CUresult (*MemGetAddressRange)(CUdeviceptr*, size_t*, CUdeviceptr) = nullptr;
  CUresult (*OccupancyMaxActiveBlocksPerMultiprocessor)(int*, CUfunction, int, size_t) = nullptr;
  bool ok = false;
};

template <class F>
void entry(const char* name, F* fn) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  cuda_check(cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q), name);
  if (q != cudaDriverEntryPointSuccess || !p) fail(rescclCudaError, std::string("driver entry point ") + name);
  *fn = (F)p;
}

Driver& driver() {
  static Driver d;
  static std::once_flag once;
  std::call_once(once, [] {
    try {
      entry("cuModuleLoadData", &d.ModuleLoadData);
      entry("cuModuleGetFunction", &d.ModuleGetFunction);
      entry("cuModuleUnload", &d.ModuleUnload);
      entry("cuLaunchCooperativeKernel", &d.LaunchCooperativeKernel);
      entry("cuLaunchKernel", &d.LaunchKernel);
      entry("cuGetErrorString", &d.GetErrorString);
      entry("cuFuncSetAttribute", &d.FuncSetAttribute);
      entry("cuMemGetAddressRange", &d.MemGetAddressRange);
      entry("cuOccupancyMaxActiveBlocksPerMultiprocessor", &d.OccupancyMaxActiveBlocksPerMultiprocessor);
      d.ok = true;
    } catch (Error&) {
      d.ok = false;
    }
  });
  if (!d.ok) fail(rescclCudaError, "CUDA driver entry points unavailable (no GPU / driver?)");
  return d;
}

void cu_check(CUresult r, const char* what) {
  if (r != CUDA_SUCCESS) {
    const char* s = "?";
    if (driver().GetErrorString) driver().GetErrorString(r, &s);
    fail(rescclCudaError, std::string(what) + ": " + s);
  }
}

// ---------------------------------------------------------------- options
struct Options {
  int instances = 1;
  int64_t chunk_bytes = 1 << 20;  // Table 2
  int fifo_depth = 4;
  int nwarps = 16;                // Table 2
  LinkModel model = LinkModel::Pair;
  bool model_set = false;  // linkmodel given explicitly (a TB budget then keeps it)
  bool fuse = true;
  int tb_budget = 0;
  int tma = 1;
  int tma_tile = 24576;   // r01 geometry sweeps: the engine costs per tile, so 24 KiB x 2 stages per lane
                          // (192 KiB smem per CTA, one CTA per SM) moves 1.4x the bytes per SM of 12 KiB x 4
  int tma_stages = 2;
  int trace = 0;
  int phase = 0;     // %globaltimer phase records per (primitive, micro-batch) (rescclGetPhaseTrace)
  int relay_bypass = 1;  // DESIGN R29: dependents of a flags-only push receive wait on its flag
  int lookahead = 1;     // DESIGN R30: "writable" credits posted ahead of the lane (1: TMA variant, 2: both)
  int sched = 0;     // 0 = HPDS (Alg. 1), 1 = round-robin baseline
  int direct = 0;    // direct transport (R23): virtual ranks / single-process only
  int pushreduce = 0;  // with direct: rrc tasks keep the staged FIFO -- push-reduce (R31)
  int l2hint = 1;
  int tma_min = 32768;   // r01 (24 KiB tiles): the TMA engine wins from 32 KiB slices (16 MiB AR +31%)
  int backoff = 1;
  int pollacq = 0;
  int jitter = 0;
  int prefetch = 0;  // r01: L2 prefetch evicts FIFO lines and loses 10-25%
  int pool_cap = 0;  // stages of the CTA pool one lane may hold (0 = all)
  int ring = 0;      // lane-private TMA stage rings (1) vs one pool shared by both lanes (0)
  int devepoch = 1;  // device-side flag epochs (graph-capturable launches) vs host-side (0)
  int bulkred = -1;  // in-place reduce primitives: cp.reduce.async.bulk of the incoming tile
                     // (-1 = auto: on for AllReduce, where it measured +16% per SM; r01_bulkred_inplace)
  int cpoll = 0;     // combine warps: one polling warp + named barrier (1) vs all polling (0)
  int early_exit = 1;  // the lane engine leaves its loop right after the last post
  int post_group = 1;  // consecutive dependency-free pull-sends posted as one group
  int split_fence = 1;  // one-sided release / acquire fences
  int store_lag = 1; // bulk stores a lane lets drain before it blocks to reuse a stage
  int sys_rank = -1; // rescclCompileIr / rescclCodegenIr: one rank's multi-process (.sys) kernel
  int nvls = 0;      // f3: NVLS transport for calls whose buffers lie in NVLS windows
  int nvls_ctas = 16;  // CTAs (x 512 threads) per rank of an NVLS launch
  // size range this algorithm serves (bytes of the per-rank buffer S: AR count x elt, AG /
  // RS N x count x elt); a call picks the most recently loaded / activated algorithm of its
  // collective whose range holds its size (a size-based tuner over loaded schedules)
  long long min_bytes = 0;
  long long max_bytes = -1;  // -1: unbounded
};

std::map<std::string, std::string> parse_kv(const char* s) {
  std::map<std::string, std::string> kv;
  if (!s) return kv;
  std::istringstream is(s);
  std::string w;
  while (is >> w) {
    auto e = w.find('=');
    if (e == std::string::npos) fail(rescclInvalidArgument, "option '" + w + "' is not key=value");
    kv[w.substr(0, e)] = w.substr(e + 1);
  }
  return kv;
}

long to_long(const std::string& v, const std::string& k) {
  try {
    size_t p = 0;
    long x = std::stol(v, &p);
    if (p != v.size()) throw 0;
    return x;
  } catch (...) {
    fail(rescclInvalidArgument, "option " + k + " is not an integer: " + v);
  }
}

void apply_kv(Options& o, const std::string& k, const std::string& v) {
  if (k == "instances") o.instances = (int)to_long(v, k);
  else if (k == "chunkbytes") o.chunk_bytes = to_long(v, k);
  else if (k == "fifodepth") o.fifo_depth = (int)to_long(v, k);
  else if (k == "nwarps") o.nwarps = (int)to_long(v, k);
  else if (k == "fuse") o.fuse = to_long(v, k) != 0;
  else if (k == "tbbudget") o.tb_budget = (int)to_long(v, k);
  else if (k == "tma") o.tma = (int)to_long(v, k);
  else if (k == "tmatile") o.tma_tile = (int)to_long(v, k);
  else if (k == "tmastages") o.tma_stages = (int)to_long(v, k);
  else if (k == "trace") o.trace = (int)to_long(v, k);
  else if (k == "phase") o.phase = (int)to_long(v, k);
  else if (k == "relaybypass") o.relay_bypass = (int)to_long(v, k);
  else if (k == "lookahead") o.lookahead = (int)to_long(v, k);
  else if (k == "l2hint") o.l2hint = (int)to_long(v, k);
  else if (k == "prefetch") o.prefetch = (int)to_long(v, k);
  else if (k == "tmamin") o.tma_min = (int)to_long(v, k);
  else if (k == "direct") o.direct = (int)to_long(v, k);
  else if (k == "pushreduce") o.pushreduce = (int)to_long(v, k);
  else if (k == "backoff") o.backoff = (int)to_long(v, k);
  else if (k == "pollacq") o.pollacq = (int)to_long(v, k);
  else if (k == "jitter") o.jitter = (int)to_long(v, k);
  else if (k == "sysrank") o.sys_rank = (int)to_long(v, k);
  else if (k == "poolcap") o.pool_cap = (int)to_long(v, k);
  else if (k == "storelag") o.store_lag = (int)to_long(v, k);
  else if (k == "splitfence") o.split_fence = (int)to_long(v, k);
  else if (k == "postgroup") o.post_group = (int)to_long(v, k);
  else if (k == "earlyexit") o.early_exit = (int)to_long(v, k);
  else if (k == "ring") o.ring = (int)to_long(v, k);
  else if (k == "cpoll") o.cpoll = (int)to_long(v, k);
  else if (k == "bulkred") o.bulkred = (int)to_long(v, k);
  else if (k == "devepoch") o.devepoch = (int)to_long(v, k);
  else if (k == "nvls") o.nvls = (int)to_long(v, k);
  else if (k == "nvlsctas") o.nvls_ctas = (int)to_long(v, k);
  else if (k == "minbytes") o.min_bytes = to_long(v, k);
  else if (k == "maxbytes") o.max_bytes = to_long(v, k);
  else if (k == "sched") {
    if (v == "hpds") o.sched = 0;
    else if (v == "rr") o.sched = 1;
    else fail(rescclInvalidArgument, "sched must be hpds|rr");
  }
  else if (k == "linkmodel") {
    if (v == "pair") o.model = LinkModel::Pair;
    else if (v == "port") o.model = LinkModel::Port;
    else fail(rescclInvalidArgument, "linkmodel must be pair|port");
    o.model_set = true;
  }
}

Options make_options(const Ir& ir, const char* extra) {
  Options o;
  o.nwarps = ir.nwarps;
  for (auto& kv : ir.extra) apply_kv(o, kv.first, kv.second);
  static const std::pair<const char*, const char*> envs[] = {
      {"RESCCL_INSTANCES", "instances"}, {"RESCCL_CHUNK_BYTES", "chunkbytes"}, {"RESCCL_FIFO_DEPTH", "fifodepth"},
      {"RESCCL_NWARPS", "nwarps"},       {"RESCCL_LINK_MODEL", "linkmodel"},   {"RESCCL_FUSE", "fuse"},
      {"RESCCL_TB_BUDGET", "tbbudget"}, {"RESCCL_TMA", "tma"}, {"RESCCL_TMA_TILE", "tmatile"},
      {"RESCCL_TMA_STAGES", "tmastages"}, {"RESCCL_TRACE", "trace"}, {"RESCCL_L2HINT", "l2hint"}, {"RESCCL_PREFETCH", "prefetch"}, {"RESCCL_SCHED", "sched"}, {"RESCCL_TMA_MIN", "tmamin"}, {"RESCCL_DIRECT", "direct"}, {"RESCCL_BACKOFF", "backoff"}, {"RESCCL_POLL_ACQ", "pollacq"}, {"RESCCL_JITTER", "jitter"}, {"RESCCL_RING", "ring"}, {"RESCCL_STORE_LAG", "storelag"}, {"RESCCL_SPLIT_FENCE", "splitfence"}, {"RESCCL_POST_GROUP", "postgroup"}, {"RESCCL_EARLY_EXIT", "earlyexit"}, {"RESCCL_NVLS", "nvls"}, {"RESCCL_CPOLL", "cpoll"}, {"RESCCL_BULKRED", "bulkred"}, {"RESCCL_DEVEPOCH", "devepoch"}, {"RESCCL_NVLS_CTAS", "nvlsctas"}};
  for (auto& e : envs)
    if (const char* v = getenv(e.first)) apply_kv(o, e.second, v);
  for (auto& kv : parse_kv(extra)) apply_kv(o, kv.first, kv.second);
  if (o.instances < 1 || o.instances > 64) fail(rescclInvalidArgument, "instances must be 1..64");
  if (o.fifo_depth < 1 || o.fifo_depth > 64) fail(rescclInvalidArgument, "fifodepth must be 1..64");
  if (o.chunk_bytes < 256 || o.chunk_bytes > (1ll << 30)) fail(rescclInvalidArgument, "chunkbytes out of range");
  if (o.nwarps < 2 || o.nwarps > 32 || o.nwarps % 2) fail(rescclInvalidArgument, "nwarps must be even, 2..32");
  // the TMA lane engine needs combine warps beside each lane's leader warp: a one-warp lane
  // (nwarps=2, the smallest CTAs, for small messages) always takes the register path
  if (o.nwarps < 4) o.tma = 0;
  if (o.tma_tile < 1024 || o.tma_tile % 128 || o.tma_stages < 1 || o.tma_stages > 8 ||
      4 * o.tma_tile * o.tma_stages > 224 * 1024)
    fail(rescclInvalidArgument, "tmatile must be a multiple of 128 >= 1024, tmastages 1..8, 4*tile*stages <= 224 KiB");
  if (o.nvls_ctas < 1 || o.nvls_ctas > 148) fail(rescclInvalidArgument, "nvlsctas must be 1..148");
  if (o.bulkred < 0) o.bulkred = ir.coll == Coll::AllReduce ? 1 : 0;
  if (o.store_lag < 1 || o.store_lag > o.tma_stages)
    fail(rescclInvalidArgument, "storelag must be 1..tmastages");
  return o;
}

// Plan an IR under the options.  A TB budget B picks the link
// model and the instance count: instances = floor(B / T_min) under the pair model;
// below T_min the port model (one duplex CTA per rank) with B instances.
Plan lower_with(const Ir& ir, LinkModel m, const Options& o) {
  if (o.sched == 1) {
    Dag d = build_dag(ir);
    auto pr = round_robin(ir, d, m);
    return lower(ir, m, o.fuse, &pr, o.direct != 0, o.pushreduce != 0);
  }
  return lower(ir, m, o.fuse, nullptr, o.direct != 0, o.pushreduce != 0);
}

Plan make_plan(const Ir& ir, Options& o) {
  if (o.tb_budget > 0 && o.model_set && o.model == LinkModel::Port) {
    // explicit port model under a TB budget: one duplex CTA per rank x B instances
    Plan q = lower_with(ir, LinkModel::Port, o);
    int t1 = 1;
    for (auto& r : q.ranks) t1 = std::max(t1, (int)r.ctas.size());
    o.instances = std::max(1, o.tb_budget / t1);
    return q;
  }
  if (o.tb_budget > 0) {
    Plan p = lower_with(ir, LinkModel::Pair, o);
    int tmin = 1;
    for (auto& r : p.ranks) tmin = std::max(tmin, (int)r.ctas.size());
    if (o.tb_budget >= tmin) {
      o.model = LinkModel::Pair;
      o.instances = std::max(1, o.tb_budget / tmin);
      return p;
    }
    o.model = LinkModel::Port;
    Plan q = lower_with(ir, LinkModel::Port, o);
    int t1 = 1;
    for (auto& r : q.ranks) t1 = std::max(t1, (int)r.ctas.size());
    o.instances = std::max(1, o.tb_budget / t1);
    return q;
  }
  return lower_with(ir, o.model, o);
}

Plan plan_checked(const Ir& ir, Options& o) {
  Plan p = make_plan(ir, o);
  std::string why;
  for (int nmb : {1, 2, 3})
    if (!deadlock_free(p, 1, nmb, &why)) fail(rescclInvalidUsage, "plan deadlocks: " + why);
  return p;
}

int elt_size(rescclDataType_t t) {
  switch (t) {
    case rescclInt32: case rescclFloat32: return 4;
    case rescclFloat16: case rescclBfloat16: return 2;
  }
  return 0;
}
const char* dtype_tag(rescclDataType_t t) {
  switch (t) {
    case rescclInt32: return "rdev::TI32";
    case rescclFloat32: return "rdev::TF32";
    case rescclFloat16: return "rdev::TF16";
    case rescclBfloat16: return "rdev::TBF16";
  }
  return "?";
}

// ---------------------------------------------------------------- NVRTC
std::vector<char> nvrtc_compile(const std::string& gen_src, rescclDataType_t dt, rescclRedOp_t op, bool gpu_scope,
                                std::string* log_out = nullptr) {
  const char* hdrs[] = {kDeviceSrc};
  const char* hdr_names[] = {"resccl_device.cuh"};
  nvrtcProgram prog;
  if (nvrtcCreateProgram(&prog, gen_src.c_str(), "resccl_gen.cu", 1, hdrs, hdr_names) != NVRTC_SUCCESS)
    fail(rescclCudaError, "nvrtcCreateProgram failed");
  std::string dT = std::string("-DRESCCL_T=") + dtype_tag(dt);
  std::string dO = "-DRESCCL_OP=" + std::to_string((int)op);
  std::vector<const char*> opts = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo", dT.c_str(), dO.c_str(),
                                   "-DRESCCL_MAXR=32"};
  nvrtcResult rc = nvrtcCompileProgram(prog, (int)opts.size(), opts.data());
  size_t logsz = 0;
  nvrtcGetProgramLogSize(prog, &logsz);
  std::string log(logsz, '\0');
  if (logsz) nvrtcGetProgramLog(prog, &log[0]);
  if (log_out) *log_out = log;
  if (rc != NVRTC_SUCCESS) {
    nvrtcDestroyProgram(&prog);
    fail(rescclCudaError, std::string("NVRTC: ") + nvrtcGetErrorString(rc) + "\n" + log.substr(0, 4000));
  }
  size_t n = 0;
  nvrtcGetCUBINSize(prog, &n);
  std::vector<char> cubin(n);
  nvrtcGetCUBIN(prog, cubin.data());
  nvrtcDestroyProgram(&prog);
  return cubin;
}

// ---------------------------------------------------------------- algorithm state
struct Kern {
  CUmodule mod = nullptr;
  CUfunction fn = nullptr;
  int smem = 0;
  int max_grid = -1;  // co-resident blocks (cooperative launch limit), per block size
  int max_grid_block = 0;
};

struct AlgoShared {
  std::string text;
  Ir ir;
  Options opt;
  Plan plan;
  Layout lay;
  std::string json;
  unsigned long long mb_cum = 0;       // virtual group: one counter for all ranks
  unsigned long long* dev_epochs = nullptr;  // virtual group: device-side epochs (devepoch=1)
  std::map<std::string, Kern> kernels;  // key: dtype/op/ranks/scope
  std::vector<char*> region;           // virtual group: per-rank plan region (one allocation)
  unsigned long long* trace_host = nullptr;  // RESCCL_TRACE buffer (host-mapped)
  unsigned long long* trace_dev = nullptr;
  int trace_blocks = 0;                // blocks covered by the last traced launch
  int trace_block_base = 0;
  unsigned long long* phase_dev = nullptr;  // phase=1: records of the last launch (device memory)
  int phase_blocks = 0, phase_block_base = 0, phase_dev_id = 0;
  std::shared_ptr<AlgoShared> twin;    // multi-process direct plan: staged plan for unregistered buffers
  char* region_alloc = nullptr;
  int64_t region_off = 0;              // multi-process: offset inside the arena
};

}  // namespace

struct rescclAlgo {
  std::shared_ptr<AlgoShared> s;
  rescclComm* comm = nullptr;
  unsigned long long mb_cum = 0;       // multi-process: this rank's counter
  unsigned long long twin_mb_cum = 0;  // ... and its staged twin's
  unsigned long long epoch = 0;        // direct calls issued (exit-barrier target)
  unsigned long long* dev_epochs[2] = {nullptr, nullptr};  // multi-process: device epochs (plan, twin)
};

namespace {
struct Group;
struct NvlsWin;
}

// copy streams and events of host-buffer collectives (upload, download)
struct HostCopy {
  cudaStream_t h2d = nullptr, d2h = nullptr;
  std::vector<cudaEvent_t> ev;
  void release() {
    for (auto e : ev) cudaEventDestroy(e);
    ev.clear();
    if (h2d) cudaStreamDestroy(h2d);
    if (d2h) cudaStreamDestroy(d2h);
    h2d = d2h = nullptr;
  }
};

struct rescclComm {
  int rank = 0, nranks = 1, dev = 0;
  bool connected = false;
  int mode = 0;  // 0 multi-process (IPC), 1 virtual (shared device), 2 single-process multi-device
  Group* group = nullptr;
  char* arena = nullptr;
  size_t arena_bytes = 0, arena_used = 0;
  std::vector<char*> peer_arena;  // size nranks (self = arena)
  std::vector<bool> peer_opened;
  int* err_host = nullptr;
  int* err_dev = nullptr;
  std::vector<std::unique_ptr<rescclAlgo>> algos;
  rescclAlgo* active[3] = {nullptr, nullptr, nullptr};
  std::vector<rescclAlgo*> ranked[3];  // per collective, activation order (most recent last)
  char* scratch = nullptr;
  size_t scratch_bytes = 0;
  std::vector<rescclComm*> peers_local;  // mode 2: every comm of the process
  // registered symmetric windows (multi-process direct transport): local range and every
  // peer's corresponding range as mapped in this process
  struct Window {
    char* base = nullptr;
    size_t bytes = 0;
    std::vector<char*> peer;
  };
  std::vector<Window> windows;
  std::map<std::string, char*> ipc_maps;  // opened peer allocations (handle bytes -> mapped base)
  std::vector<std::shared_ptr<NvlsWin>> nvls;  // f3: this rank's NVLS windows (multicast-bound)
  // host-buffer collectives: device staging (send and receive regions) of this rank
  char* hstage = nullptr;
  size_t hstage_bytes = 0;
  HostCopy hcopy;  // host-buffer collectives: copy streams (multi-process / multi-device)
  // host-buffer piece size (RESCCL_HOST_PIECE), fixed at creation; multi-process ranks
  // check at connect that every rank uses the same value (the piece schedule decides the
  // launches every rank must issue alike)
  size_t host_piece = 0;
  std::vector<char*> retired_scratch;  // scratch buffers replaced by larger ones (freed at destroy)
};

namespace {

struct Pending {
  int coll;
  size_t count;
  int dtype, op;
  int arrived = 0;
  AlgoShared* algo = nullptr;
  std::vector<const void*> send;
  std::vector<void*> recv;
  std::vector<cudaStream_t> streams;
  bool host = false;  // some rank passed a host buffer (staged by group_host_launch)
};

struct Group {
  int dev = 0, nranks = 0;
  std::vector<rescclComm*> comms;
  std::map<std::string, std::shared_ptr<AlgoShared>> algos;  // by IR text + opts
  std::vector<unsigned long long> issued;                   // per rank: collectives issued
  std::deque<Pending> pending;                               // pending[0] = sequence `base`
  unsigned long long base = 0;
  int* err_host = nullptr;
  int* err_dev = nullptr;
  std::vector<cudaEvent_t> events;
  HostCopy hcopy;  // host-buffer collectives of the group
  int refs = 0;
};

unsigned long long timeout_ns() {
  const char* v = getenv("RESCCL_TIMEOUT_MS");
  long ms = v ? atol(v) : 30000;
  if (ms <= 0) ms = 30000;
  return (unsigned long long)ms * 1000000ull;
}

size_t arena_default() {
  const char* v = getenv("RESCCL_ARENA_BYTES");
  return v ? (size_t)atoll(v) : (size_t)128 << 20;
}

// IR text, or a ResCCLang program (`def ResCCLAlgo(...):`, Fig. 14/16)
Ir parse_any(const std::string& text) {
  std::istringstream is(text);
  std::string line;
  while (std::getline(is, line)) {  // first non-blank, non-comment line decides
    size_t i = line.find_first_not_of(" \t\r");
    if (i == std::string::npos || line[i] == '#') continue;
    if (line.compare(i, 4, "def ") == 0) return parse_rescclang(text);
    break;
  }
  return parse_ir(text);
}

std::shared_ptr<AlgoShared> build_algo(const std::string& text, int nranks, const char* extra = nullptr) {
  auto a = std::make_shared<AlgoShared>();
  a->text = text;
  try {
    a->ir = parse_any(text);
  } catch (PlanError& e) {
    fail(rescclInvalidUsage, std::string("IR: ") + e.what());
  }
  if (a->ir.nranks != nranks)
    fail(rescclInvalidUsage, "IR nranks=" + std::to_string(a->ir.nranks) + " != communicator size " +
                                 std::to_string(nranks));
  if (nranks > kMaxR) fail(rescclInvalidUsage, "at most 32 ranks per communicator");
  try {
    a->opt = make_options(a->ir, extra);
    a->plan = plan_checked(a->ir, a->opt);
    a->lay = make_layout(a->plan, a->opt.fifo_depth, a->opt.instances, a->opt.chunk_bytes);
  } catch (PlanError& e) {
    fail(rescclInvalidUsage, std::string("plan: ") + e.what());
  }
  return a;
}

std::string info_json(const AlgoShared& a) {
  std::ostringstream o;
  std::string pj = plan_json(a.plan);
  o << "{\"plan\":" << pj << ",\"instances\":" << a.opt.instances << ",\"chunkbytes\":" << a.opt.chunk_bytes
    << ",\"fifodepth\":" << a.opt.fifo_depth << ",\"nwarps\":" << a.opt.nwarps << ",\"tma\":" << a.opt.tma
    << ",\"tmatile\":" << a.opt.tma_tile << ",\"tmastages\":" << a.opt.tma_stages << ",\"l2hint\":" << a.opt.l2hint << ",\"prefetch\":" << a.opt.prefetch << ",\"sched\":\""
    << (a.opt.sched ? "rr" : "hpds") << "\",\"direct\":" << a.opt.direct << ",\"pushreduce\":" << a.opt.pushreduce << ",\"bulkred\":" << a.opt.bulkred << ",\"devepoch\":" << a.opt.devepoch << ",\"nvls\":" << a.opt.nvls << ",\"nvlsctas\":" << a.opt.nvls_ctas << ",\"linkmodel\":\""
    << (a.opt.model == LinkModel::Pair ? "pair" : "port") << "\",\"region_bytes\":" << a.lay.region_bytes
    << ",\"ctas\":[";
  for (size_t r = 0; r < a.lay.ctas.size(); ++r) o << (r ? "," : "") << a.lay.ctas[r];
  o << "],\"blocks_per_rank\":[";
  for (size_t r = 0; r < a.lay.ctas.size(); ++r) o << (r ? "," : "") << a.lay.ctas[r] * a.opt.instances;
  o << "]}";
  return o.str();
}

// use_tma: the call's instance slices reach `tmamin` bytes; otherwise a variant without
// the TMA engine (no dynamic shared memory, no mbarrier setup) is launched -- small
// messages are latency-bound and the staging only costs launch overhead there.
// codegen options carried by an Options set (every kernel-build path uses this)
CodegenOpts codegen_opts(const Options& o) {
  CodegenOpts co;
  co.nwarps = o.nwarps;
  co.tma = o.tma;
  co.tma_tile = o.tma_tile;
  co.tma_stages = o.tma_stages;
  co.trace = o.trace;
  co.phase = o.phase;
  co.relay_bypass = o.relay_bypass;
  co.lookahead = o.lookahead;
  co.l2hint = o.l2hint;
  co.prefetch = o.prefetch;
  co.tma_min = o.tma_min;
  co.backoff = o.backoff;
  co.pollacq = o.pollacq;
  co.jitter = o.jitter;
  co.pool_cap = o.pool_cap;
  co.store_lag = o.store_lag;
  co.split_fence = o.split_fence;
  co.post_group = o.post_group;
  co.early_exit = o.early_exit;
  co.ring = o.ring;
  co.cpoll = o.cpoll;
  co.bulkred = o.bulkred;
  return co;
}

Kern& get_kernel(AlgoShared& a, rescclDataType_t dt, rescclRedOp_t op, int lo, int hi, bool gpu_scope,
                 bool use_tma) {
  std::string key = std::to_string((int)dt) + "/" + std::to_string((int)op) + "/" + std::to_string(lo) + "-" +
                    std::to_string(hi) + "/" + (gpu_scope ? "g" : "s") + (use_tma ? "/t" : "/n");
  auto it = a.kernels.find(key);
  if (it != a.kernels.end()) return it->second;
  CodegenOpts co = codegen_opts(a.opt);
  co.rank_lo = lo;
  co.rank_hi = hi;
  co.gpu_scope = gpu_scope;
  co.tma = use_tma ? a.opt.tma : 0;
  // writable lookahead (R30): 1 = in the TMA-engine variant only (large slices, where it
  // measured +2-4% at 16-64 MiB; in the latency-bound register-path variant its extra
  // probes and fences cost more than the early credits save), 2 = in both variants
  co.lookahead = a.opt.lookahead >= 2 || (a.opt.lookahead == 1 && use_tma) ? 1 : 0;
  co.exit_barrier = a.opt.direct && !gpu_scope;
  std::string src = codegen(a.plan, a.lay, co);
  if (const char* dump = getenv("RESCCL_DUMP_SRC")) {  // debugging aid: write the generated source
    if (FILE* f = fopen((std::string(dump) + "_" + a.ir.name + "_" + coll_name(a.ir.coll) + ".cu").c_str(), "w")) {
      fputs(src.c_str(), f);
      fclose(f);
    }
  }
  std::vector<char> cubin = nvrtc_compile(src, dt, op, gpu_scope);
  Kern k;
  cu_check(driver().ModuleLoadData(&k.mod, cubin.data()), "cuModuleLoadData");
  cu_check(driver().ModuleGetFunction(&k.fn, k.mod, "resccl_kernel"), "cuModuleGetFunction");
  k.smem = codegen_smem_bytes(co);
  if (k.smem > 0)
    cu_check(driver().FuncSetAttribute(k.fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, k.smem),
             "cuFuncSetAttribute");
  return a.kernels[key] = k;
}

void set_err(const Error& e) { g_last_error = e.msg; }

#define API_BEGIN try {
#define API_END                                      \
  }                                                  \
  catch (Error & e) {                                \
    set_err(e);                                      \
    return e.code;                                   \
  }                                                  \
  catch (PlanError & e) {                            \
    g_last_error = e.what();                         \
    return rescclInvalidUsage;                       \
  }                                                  \
  catch (std::exception & e) {                       \
    g_last_error = e.what();                         \
    return rescclInternalError;                      \
  }                                                  \
  catch (...) {                                      \
    g_last_error = "unknown exception";              \
    return rescclInternalError;                      \
  }                                                  \
  return rescclSuccess;

void write_out(const std::string& s, void* buf, size_t* len) {
  if (!len) fail(rescclInvalidArgument, "len is NULL");
  if (!buf) {
    *len = s.size() + 1;
    return;
  }
  if (*len < s.size() + 1) {
    size_t need = s.size() + 1;
    *len = need;
    fail(rescclInvalidArgument, "buffer too small (need " + std::to_string(need) + " bytes)");
  }
  memcpy(buf, s.c_str(), s.size() + 1);
  *len = s.size() + 1;
}

void alloc_err_word(int** host, int** dev) {
  cuda_check(cudaHostAlloc((void**)host, 64, cudaHostAllocMapped | cudaHostAllocPortable), "cudaHostAlloc");
  memset(*host, 0, 64);
  cuda_check(cudaHostGetDevicePointer((void**)dev, *host, 0), "cudaHostGetDevicePointer");
}

// ---------------------------------------------------------------- launching
struct CallDesc {
  int coll;
  size_t count;
  rescclDataType_t dt;
  rescclRedOp_t op;
};

Geometry call_geometry(const AlgoShared& a, const CallDesc& c) {
  return geometry(a.ir.coll, a.ir.nranks, (int64_t)c.count, elt_size(c.dt), a.opt.chunk_bytes, a.opt.instances);
}

void ensure_scratch(rescclComm* comm, size_t bytes, cudaStream_t s = nullptr) {
  if (comm->scratch_bytes >= bytes) return;
  // growing allocates: not allowed inside a CUDA-graph capture (the capture would be
  // invalidated) -- the first ReduceScatter of a size must run eagerly before capturing
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  if (s && cudaStreamIsCapturing(s, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone)
    fail(rescclInvalidUsage, "ReduceScatter scratch would grow during CUDA-graph capture: run one call of this "
                             "size (or larger) eagerly before capturing");
  cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
  char* p = nullptr;
  cuda_check(cudaMalloc((void**)&p, bytes), "cudaMalloc(scratch)");
  // the old buffer may still be in use by queued kernels: keep it until rescclCommDestroy
  if (comm->scratch) comm->retired_scratch.push_back(comm->scratch);
  comm->scratch = p;
  comm->scratch_bytes = bytes;
}

void launch(Kern& k, int grid, int block, KArgs& args, cudaStream_t s) {
  // every CTA of a schedule must be co-resident (they wait on each other): check before
  // the cooperative launch so the error names the cause
  if (k.max_grid < 0 || k.max_grid_block != block) {
    int per_sm = 0, dev = 0, nsm = 0;
    cu_check(driver().OccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k.fn, block, (size_t)k.smem),
             "cuOccupancyMaxActiveBlocksPerMultiprocessor");
    cuda_check(cudaGetDevice(&dev), "cudaGetDevice");
    cuda_check(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev), "cudaDeviceGetAttribute");
    k.max_grid = per_sm * nsm;
    k.max_grid_block = block;
  }
  if (grid > k.max_grid)
    fail(rescclInvalidUsage, "the plan needs " + std::to_string(grid) + " co-resident CTAs (CTAs per rank x "
                             "instances x ranks on this device) but at most " + std::to_string(k.max_grid) +
                             " fit: lower instances / nwarps / the TB budget");
  void* params[] = {&args};
  // cooperative launch: the driver schedules the grid only when every CTA can be resident
  // (a plain launch could start part of the grid beside a concurrent compute kernel, whose
  // CTAs would then wait on CTAs not yet running).  RESCCL_COOP=0 (measurement aid) uses a
  // plain launch.
  static const bool coop = [] {
    const char* v = getenv("RESCCL_COOP");
    return !(v && v[0] == '0');
  }();
  if (coop)
    cu_check(driver().LaunchCooperativeKernel(k.fn, grid, 1, 1, block, 1, 1, k.smem, (CUstream)s, params),
             "cuLaunchCooperativeKernel");
  else
    cu_check(driver().LaunchKernel(k.fn, grid, 1, 1, block, 1, 1, k.smem, (CUstream)s, params, nullptr),
             "cuLaunchKernel");
}

void fill_geometry(KArgs& ka, const Geometry& g, size_t count) {
  ka.count = (long long)count;
  ka.C = g.C;
  ka.M = g.M;
  ka.Mi = g.Mi;
  ka.n_mb = g.n_mb;
}

unsigned long long* trace_buffer(AlgoShared& a, int blocks, int block_base) {
  if (!a.opt.trace) return nullptr;
  if (!a.trace_host) {
    size_t bytes = (size_t)a.lay.total_pairs * a.opt.instances * 2 * 8 * sizeof(unsigned long long);
    cuda_check(cudaHostAlloc((void**)&a.trace_host, bytes, cudaHostAllocMapped | cudaHostAllocPortable),
               "cudaHostAlloc(trace)");
    memset(a.trace_host, 0, bytes);
    cuda_check(cudaHostGetDevicePointer((void**)&a.trace_dev, a.trace_host, 0), "cudaHostGetDevicePointer");
  }
  a.trace_blocks = blocks;
  a.trace_block_base = block_base;
  return a.trace_dev;
}

// phase=1: the record area of this launch, cleared on the launch stream
unsigned long long* phase_buffer(AlgoShared& a, int blocks, int block_base, int dev, cudaStream_t s) {
  if (!a.opt.phase) return nullptr;
  const size_t per = (size_t)RESCCL_PH_MAX_HOST * 8 * sizeof(unsigned long long);
  const size_t bytes = (size_t)a.lay.total_pairs * a.opt.instances * 2 * per;
  if (!a.phase_dev) cuda_check(cudaMalloc((void**)&a.phase_dev, bytes), "cudaMalloc(phase)");
  cuda_check(cudaMemsetAsync(a.phase_dev, 0, bytes, s), "cudaMemsetAsync(phase)");
  a.phase_blocks = blocks;
  a.phase_block_base = block_base;
  a.phase_dev_id = dev;
  return a.phase_dev;
}

// connected window containing [p, p + bytes), or -1
int find_window(const rescclComm* comm, const void* p, size_t bytes) {
  for (size_t w = 0; w < comm->windows.size(); ++w) {
    const auto& W = comm->windows[w];
    bool connected = true;
    for (char* q : W.peer) connected = connected && q;
    if (connected && (const char*)p >= W.base && (const char*)p + bytes <= W.base + W.bytes) return (int)w;
  }
  return -1;
}

// multi-process / multi-device path: this rank alone

void launch_rank(rescclComm* comm, rescclAlgo* algo, const CallDesc& c, const void* send, void* recv,
                 cudaStream_t s) {
  AlgoShared* ap = algo->s.get();
  unsigned long long* mb_cum = &algo->mb_cum;
  int ws = -1, wr = -1;
  if (ap->opt.direct && comm->mode == 0) {
    // direct transport across processes needs both buffers in registered symmetric
    // windows (same window and offset on every rank); otherwise the staged twin runs
    const size_t e = elt_size(c.dt);
    const size_t sb = c.count * e * (c.coll == (int)Coll::ReduceScatter ? comm->nranks : 1);
    const size_t rb = c.count * e * (c.coll == (int)Coll::AllGather ? comm->nranks : 1);
    ws = find_window(comm, send, sb);
    wr = find_window(comm, recv, rb);
    if (ws < 0 || wr < 0 || c.coll == (int)Coll::ReduceScatter) {
      ap = ap->twin.get();
      mb_cum = &algo->twin_mb_cum;
      ws = wr = -1;
    }
  }
  AlgoShared& a = *ap;
  Geometry g = call_geometry(a, c);
  if (g.n_mb == 0) return;
  cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
  KArgs ka;
  memset(&ka, 0, sizeof(ka));
  for (int q = 0; q < comm->nranks; ++q) ka.arena[q] = comm->peer_arena[q] + a.region_off;
  ka.sendbuf[comm->rank] = (const char*)send;
  ka.recvbuf[comm->rank] = (char*)recv;
  if (ws >= 0) {
    const auto& WS = comm->windows[ws];
    const auto& WR = comm->windows[wr];
    const size_t os = (const char*)send - WS.base, orr = (char*)recv - WR.base;
    for (int q = 0; q < comm->nranks; ++q) {
      ka.sendbuf[q] = WS.peer[q] + os;
      ka.recvbuf[q] = WR.peer[q] + orr;
    }
  }
  if (a.ir.coll == Coll::ReduceScatter) {
    ensure_scratch(comm, c.count * comm->nranks * elt_size(c.dt), s);
    ka.scratch[comm->rank] = comm->scratch;
  }
  fill_geometry(ka, g, c.count);
  ka.mb_base = *mb_cum;
  if (ws >= 0) ka.epoch = algo->epoch++;
  ka.block_base = a.lay.pair_start[comm->rank] * a.opt.instances;
  ka.err = comm->err_dev;
  ka.timeout_ns = timeout_ns();
  ka.trace = trace_buffer(a, a.lay.ctas[comm->rank] * a.opt.instances, ka.block_base);
  ka.phase = phase_buffer(a, a.lay.ctas[comm->rank] * a.opt.instances, ka.block_base, comm->dev, s);
  if (a.opt.devepoch) ka.epochs = algo->dev_epochs[ap == algo->s.get() ? 0 : 1];
  const bool use_tma = a.opt.tma && g.Mi * elt_size(c.dt) >= a.opt.tma_min;
  Kern& k = get_kernel(a, c.dt, c.op, comm->rank, comm->rank + 1, false, use_tma);
  launch(k, a.lay.ctas[comm->rank] * a.opt.instances, 32 * a.opt.nwarps, ka, s);
  *mb_cum += (unsigned long long)g.n_mb;
}

// virtual group: all ranks in one kernel, when the last rank arrives
void group_launch(Group* G, Pending& p) {
  AlgoShared& a = *p.algo;
  CallDesc c{p.coll, p.count, (rescclDataType_t)p.dtype, (rescclRedOp_t)p.op};
  Geometry g = call_geometry(a, c);
  if (g.n_mb == 0) return;
  cuda_check(cudaSetDevice(G->dev), "cudaSetDevice");
  KArgs ka;
  memset(&ka, 0, sizeof(ka));
  for (int q = 0; q < G->nranks; ++q) {
    ka.arena[q] = a.region[q];
    ka.sendbuf[q] = (const char*)p.send[q];
    ka.recvbuf[q] = (char*)p.recv[q];
    if (a.ir.coll == Coll::ReduceScatter) {
      ensure_scratch(G->comms[q], c.count * G->nranks * elt_size(c.dt), p.streams.back());
      ka.scratch[q] = G->comms[q]->scratch;
    }
  }
  fill_geometry(ka, g, c.count);
  ka.mb_base = a.mb_cum;
  ka.block_base = 0;
  ka.err = G->err_dev;
  ka.timeout_ns = timeout_ns();
  ka.trace = trace_buffer(a, a.lay.total_pairs * a.opt.instances, 0);
  ka.phase = phase_buffer(a, a.lay.total_pairs * a.opt.instances, 0, G->dev, p.streams.back());
  if (a.opt.devepoch) ka.epochs = a.dev_epochs;
  const bool use_tma = a.opt.tma && g.Mi * elt_size(c.dt) >= a.opt.tma_min;
  Kern& k = get_kernel(a, c.dt, c.op, 0, G->nranks, true, use_tma);
  cudaStream_t ls = p.streams.back();
  // order the launch after every caller's stream, and every caller's stream after it
  std::vector<cudaStream_t> others;
  for (auto s : p.streams)
    if (s != ls && std::find(others.begin(), others.end(), s) == others.end()) others.push_back(s);
  while (G->events.size() < 2 * others.size() + 1) {
    cudaEvent_t e;
    cuda_check(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "cudaEventCreate");
    G->events.push_back(e);
  }
  for (size_t i = 0; i < others.size(); ++i) {
    cuda_check(cudaEventRecord(G->events[i], others[i]), "cudaEventRecord");
    cuda_check(cudaStreamWaitEvent(ls, G->events[i], 0), "cudaStreamWaitEvent");
  }
  launch(k, a.lay.total_pairs * a.opt.instances, 32 * a.opt.nwarps, ka, ls);
  a.mb_cum += (unsigned long long)g.n_mb;
  if (!others.empty()) {
    cudaEvent_t done = G->events[others.size()];
    cuda_check(cudaEventRecord(done, ls), "cudaEventRecord");
    for (auto s : others) cuda_check(cudaStreamWaitEvent(s, done, 0), "cudaStreamWaitEvent");
  }
}


// ------------------------------------------------------------ host-buffer collectives
// A send or receive buffer in host memory (pinned, or pageable at pageable-copy speed) is
// staged through device memory the communicator owns: upload on a copy stream, the
// collective on the caller's stream, download on a second copy stream.  A call is cut
// into pieces of RESCCL_HOST_PIECE bytes per rank (default 32 MiB; layout at Staging) so
// that piece k's collective and piece k-1's download overlap piece k+1's upload (PCIe is
// full duplex).  The
// caller's stream waits for the last download: stream semantics are the device path's.

// Host (pinned or pageable) vs device memory.  A pointer the runtime cannot classify is
// an error (InvalidArgument), never silently treated as host memory.
bool host_ptr(const void* p, bool* pageable = nullptr) {
  cudaPointerAttributes at;
  cudaError_t e = cudaPointerGetAttributes(&at, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    // a device address the runtime does not describe (e.g. a VMM mapping) is still device
    // memory if the driver knows its range
    CUdeviceptr base = 0;
    size_t sz = 0;
    if (driver().MemGetAddressRange(&base, &sz, (CUdeviceptr)p) == CUDA_SUCCESS && sz > 0) {
      if (pageable) *pageable = false;
      return false;
    }
    fail(rescclInvalidArgument, std::string("buffer pointer not classifiable: ") + cudaGetErrorString(e));
  }
  if (pageable) *pageable = at.type == cudaMemoryTypeUnregistered;
  return at.type == cudaMemoryTypeHost || at.type == cudaMemoryTypeUnregistered;
}

size_t host_piece_bytes() {
  const char* v = getenv("RESCCL_HOST_PIECE");
  long long b = v ? atoll(v) : (32ll << 20);
  if (b < 4096) b = 4096;
  return (size_t)b & ~(size_t)255;
}

void ensure_hstage(rescclComm* comm, size_t bytes) {
  if (comm->hstage_bytes >= bytes) return;
  cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
  if (comm->hstage) {
    cuda_check(cudaDeviceSynchronize(), "cudaDeviceSynchronize");  // queued work may use it
    cuda_check(cudaFree(comm->hstage), "cudaFree(host stage)");
    comm->hstage = nullptr;
    comm->hstage_bytes = 0;
  }
  cuda_check(cudaMalloc((void**)&comm->hstage, bytes), "cudaMalloc(host stage)");
  comm->hstage_bytes = bytes;
}

void ensure_copy(HostCopy& h, size_t nev) {
  if (!h.h2d) {
    cuda_check(cudaStreamCreateWithFlags(&h.h2d, cudaStreamNonBlocking), "cudaStreamCreate");
    cuda_check(cudaStreamCreateWithFlags(&h.d2h, cudaStreamNonBlocking), "cudaStreamCreate");
  }
  while (h.ev.size() < nev) {
    cudaEvent_t e;
    cuda_check(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "cudaEventCreate");
    h.ev.push_back(e);
  }
}

// One rank's staging.  A call is cut into pieces [lo, lo+m) of the per-rank count: AR
// pieces are contiguous; an AllGather piece's output and a ReduceScatter piece's input are
// N rows of m elements, so their stage regions are piece-major (piece k's N*m block at
// N*lo) and the strided host side moves with 2D copies.  A device-side AG output or RS
// input cannot be piece-major: such calls run as one piece.  Host in-place calls (NCCL's
// rules: AR send == recv, AG send == recv + rank*count, RS recv == send + rank*count)
// stage one region.
struct Staging {
  int coll = 0, rank = 0, N = 1;
  size_t count = 0, e = 0, sb = 0, rb = 0, need = 0;
  long long soff = -1, roff = -1;  // stage offsets of the send / receive regions (-1: caller's buffer)
  bool hs = false, hr = false, inplace = false, pieces = false;
  const char* send = nullptr;
  char* recv = nullptr;
  char* stage = nullptr;

  void plan(int coll_, int rank_, int N_, const void* send_, void* recv_, size_t count_, size_t e_) {
    coll = coll_, rank = rank_, N = N_, count = count_, e = e_;
    send = (const char*)send_, recv = (char*)recv_;
    sb = count * e * (coll == (int)Coll::ReduceScatter ? N : 1);
    rb = count * e * (coll == (int)Coll::AllGather ? N : 1);
    hs = host_ptr(send);
    hr = host_ptr(recv);
    const size_t blk = (size_t)rank * count * e;
    if (hs && hr && coll == (int)Coll::AllReduce && send == recv) {
      inplace = true, need = rb, soff = roff = 0;
    } else if (hs && hr && coll == (int)Coll::AllGather && send == recv + blk) {
      inplace = true, need = rb, roff = 0, soff = (long long)blk;
    } else if (hs && hr && coll == (int)Coll::ReduceScatter && recv == send + blk) {
      inplace = true, need = sb, soff = 0, roff = (long long)blk;
    } else {
      if (hs) soff = 0, need += sb;
      if (hr) roff = (long long)need, need += rb;
    }
    pieces = coll == (int)Coll::AllReduce || (coll == (int)Coll::AllGather ? hr : hs);
  }
  // device buffers of piece [lo, lo+m)
  const char* dsend(size_t lo, size_t m) const {
    if (coll == (int)Coll::AllGather && inplace) return drecv(lo, m) + (size_t)rank * m * e;
    const char* base = soff >= 0 ? stage + soff : send;
    return base + (coll == (int)Coll::ReduceScatter ? (size_t)N : 1) * lo * e;
  }
  char* drecv(size_t lo, size_t m) const {
    if (coll == (int)Coll::ReduceScatter && inplace) return (char*)dsend(lo, m) + (size_t)rank * m * e;
    char* base = roff >= 0 ? stage + roff : recv;
    return base + (coll == (int)Coll::AllGather ? (size_t)N : 1) * lo * e;
  }
  void upload(size_t lo, size_t m, cudaStream_t st) const {
    char* d = (char*)dsend(lo, m);
    if (coll == (int)Coll::ReduceScatter)  // N rows: host pitch count, stage pitch m
      cuda_check(cudaMemcpy2DAsync(d, m * e, send + lo * e, count * e, m * e, N, cudaMemcpyHostToDevice, st),
                 "cudaMemcpy2DAsync(H2D)");
    else
      cuda_check(cudaMemcpyAsync(d, send + lo * e, m * e, cudaMemcpyHostToDevice, st), "cudaMemcpyAsync(H2D)");
  }
  void download(size_t lo, size_t m, cudaStream_t st) const {
    const char* d = drecv(lo, m);
    if (coll == (int)Coll::AllGather)
      cuda_check(cudaMemcpy2DAsync(recv + lo * e, count * e, d, m * e, m * e, N, cudaMemcpyDeviceToHost, st),
                 "cudaMemcpy2DAsync(D2H)");
    else
      cuda_check(cudaMemcpyAsync(recv + lo * e, d, m * e, cudaMemcpyDeviceToHost, st), "cudaMemcpyAsync(D2H)");
  }
};

size_t piece_elems(const rescclComm* comm, size_t count, size_t e) {
  const size_t pb = comm->host_piece ? comm->host_piece : host_piece_bytes();
  return std::min(count, std::max<size_t>(1, pb / e));
}

// multi-process / multi-device rank
void host_rank(rescclComm* comm, rescclAlgo* algo, const CallDesc& c, const void* send, void* recv,
               cudaStream_t s) {
  const size_t e = elt_size(c.dt);
  Staging P;
  P.plan(c.coll, comm->rank, comm->nranks, send, recv, c.count, e);
  ensure_hstage(comm, P.need);
  P.stage = comm->hstage;
  const size_t pe = P.pieces ? piece_elems(comm, c.count, e) : c.count, np = (c.count + pe - 1) / pe;
  HostCopy& h = comm->hcopy;
  ensure_copy(h, 2 * np + 2);
  size_t ei = 0;
  cuda_check(cudaEventRecord(h.ev[ei], s), "cudaEventRecord");
  cuda_check(cudaStreamWaitEvent(h.h2d, h.ev[ei], 0), "cudaStreamWaitEvent");
  cuda_check(cudaStreamWaitEvent(h.d2h, h.ev[ei++], 0), "cudaStreamWaitEvent");
  for (size_t k = 0; k < np; ++k) {
    const size_t lo = k * pe, m = std::min(pe, c.count - lo);
    if (P.hs) {
      P.upload(lo, m, h.h2d);
      cuda_check(cudaEventRecord(h.ev[ei], h.h2d), "cudaEventRecord");
      cuda_check(cudaStreamWaitEvent(s, h.ev[ei++], 0), "cudaStreamWaitEvent");
    }
    launch_rank(comm, algo, CallDesc{c.coll, m, c.dt, c.op}, P.dsend(lo, m), P.drecv(lo, m), s);
    if (P.hr) {
      cuda_check(cudaEventRecord(h.ev[ei], s), "cudaEventRecord");
      cuda_check(cudaStreamWaitEvent(h.d2h, h.ev[ei++], 0), "cudaStreamWaitEvent");
      P.download(lo, m, h.d2h);
    }
  }
  if (P.hr) {
    cuda_check(cudaEventRecord(h.ev[ei], h.d2h), "cudaEventRecord");
    cuda_check(cudaStreamWaitEvent(s, h.ev[ei++], 0), "cudaStreamWaitEvent");
  }
}

// virtual group: every rank's uploads of piece k, one launch for piece k, its downloads
void group_host_launch(Group* G, Pending& p) {
  const int N = G->nranks;
  const size_t e = elt_size((rescclDataType_t)p.dtype);
  cuda_check(cudaSetDevice(G->dev), "cudaSetDevice");
  std::vector<Staging> P(N);
  bool any_hs = false, any_hr = false, pieces = true;
  for (int q = 0; q < N; ++q) {
    P[q].plan(p.coll, q, N, p.send[q], p.recv[q], p.count, e);
    ensure_hstage(G->comms[q], P[q].need);
    P[q].stage = G->comms[q]->hstage;
    any_hs |= P[q].hs;
    any_hr |= P[q].hr;
    pieces &= P[q].pieces;
  }
  const size_t pe = pieces ? piece_elems(G->comms[0], p.count, e) : p.count, np = (p.count + pe - 1) / pe;
  cudaStream_t ls = p.streams.back();
  std::vector<cudaStream_t> others;
  for (auto s : p.streams)
    if (s != ls && std::find(others.begin(), others.end(), s) == others.end()) others.push_back(s);
  HostCopy& h = G->hcopy;
  ensure_copy(h, others.size() + 2 * np + 3);
  size_t ei = 0;
  for (auto s : others) {  // the launch stream joins every caller's stream
    cuda_check(cudaEventRecord(h.ev[ei], s), "cudaEventRecord");
    cuda_check(cudaStreamWaitEvent(ls, h.ev[ei++], 0), "cudaStreamWaitEvent");
  }
  cuda_check(cudaEventRecord(h.ev[ei], ls), "cudaEventRecord");
  cuda_check(cudaStreamWaitEvent(h.h2d, h.ev[ei], 0), "cudaStreamWaitEvent");
  cuda_check(cudaStreamWaitEvent(h.d2h, h.ev[ei++], 0), "cudaStreamWaitEvent");
  for (size_t k = 0; k < np; ++k) {
    const size_t lo = k * pe, m = std::min(pe, p.count - lo);
    if (any_hs) {
      for (int q = 0; q < N; ++q)
        if (P[q].hs) P[q].upload(lo, m, h.h2d);
      cuda_check(cudaEventRecord(h.ev[ei], h.h2d), "cudaEventRecord");
      cuda_check(cudaStreamWaitEvent(ls, h.ev[ei++], 0), "cudaStreamWaitEvent");
    }
    Pending piece = p;
    piece.count = m;
    piece.host = false;
    piece.streams.assign(1, ls);
    for (int q = 0; q < N; ++q) {
      piece.send[q] = P[q].dsend(lo, m);
      piece.recv[q] = P[q].drecv(lo, m);
    }
    group_launch(G, piece);
    if (any_hr) {
      cuda_check(cudaEventRecord(h.ev[ei], ls), "cudaEventRecord");
      cuda_check(cudaStreamWaitEvent(h.d2h, h.ev[ei++], 0), "cudaStreamWaitEvent");
      for (int q = 0; q < N; ++q)
        if (P[q].hr) P[q].download(lo, m, h.d2h);
    }
  }
  if (any_hr) {
    cuda_check(cudaEventRecord(h.ev[ei], h.d2h), "cudaEventRecord");
    cuda_check(cudaStreamWaitEvent(ls, h.ev[ei++], 0), "cudaStreamWaitEvent");
  }
  cuda_check(cudaEventRecord(h.ev[ei], ls), "cudaEventRecord");  // every caller's stream after it
  for (auto s : others) cuda_check(cudaStreamWaitEvent(s, h.ev[ei], 0), "cudaStreamWaitEvent");
}

rescclAlgo* ensure_algo(rescclComm* comm, Coll coll);
rescclAlgo* select_algo(rescclComm* comm, Coll coll, long long bytes);
bool try_nvls(rescclComm* comm, const AlgoShared& a, int coll, const void* send, void* recv, size_t count,
              rescclDataType_t dt, rescclRedOp_t op, cudaStream_t s);

void collective(rescclComm* comm, int coll, const void* send, void* recv, size_t count, rescclDataType_t dt,
                rescclRedOp_t op, void* stream) {
  if (!comm) fail(rescclInvalidArgument, "comm is NULL");
  if (!comm->connected) fail(rescclInvalidUsage, "communicator not connected");
  if (elt_size(dt) == 0) fail(rescclInvalidArgument, "bad dtype");
  if ((int)op < 0 || (int)op > 2) fail(rescclInvalidArgument, "bad op");
  if (count > 0 && (!send || !recv)) fail(rescclInvalidArgument, "null buffer");
  cudaStream_t s = (cudaStream_t)stream;
  // CUDA-graph capture: the generated kernels take their flag epochs from device memory
  // (devepoch=1, default), so a captured launch replays correctly; host-side epochs
  // (devepoch=0) and the NVLS transport's arrival counts advance on the host per call, so
  // those refuse capture rather than build a graph whose replays would hang
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  const bool capturing = cudaStreamIsCapturing(s, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone;
  if (capturing && !comm->active[coll])
    fail(rescclInvalidUsage, "load an algorithm before capturing a collective into a CUDA graph");
  bool pg_send = false, pg_recv = false;
  const bool host = count > 0 && (host_ptr(send, &pg_send) | host_ptr(recv, &pg_recv));
  // one host thread drives every rank of a single-process multi-device communicator: a
  // pageable download blocks that thread until this rank's collective finishes, which
  // waits for ranks the thread has not issued yet -- refuse instead of hanging
  if (comm->mode == 2 && (pg_send || pg_recv))
    fail(rescclInvalidArgument, "pageable host buffers are not supported with single-process multi-device "
                                "communicators (pin them, e.g. cudaHostRegister / tensor.pin_memory())");
  if (capturing && host)
    fail(rescclInvalidUsage, "host buffers cannot be captured into a CUDA graph (staged copies)");
  const long long S = (long long)count * elt_size(dt) * (coll == (int)Coll::AllReduce ? 1 : comm->nranks);
  rescclAlgo* algo = select_algo(comm, (Coll)coll, S);
  if (capturing && (!algo->s->opt.devepoch || algo->s->opt.nvls))
    fail(rescclInvalidUsage, "this algorithm cannot be captured into a CUDA graph (devepoch=0 or nvls=1: "
                             "host-side epochs)");
  if (comm->mode != 1) {
    if (count == 0) return;
    if (host) {
      cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
      host_rank(comm, algo, CallDesc{coll, count, dt, op}, send, recv, s);
      return;
    }
    if (algo->s->opt.nvls && try_nvls(comm, *algo->s, coll, send, recv, count, dt, op, s)) return;
    launch_rank(comm, algo, CallDesc{coll, count, dt, op}, send, recv, s);
    return;
  }
  Group* G = comm->group;
  unsigned long long seq = G->issued[comm->rank]++;
  if (seq < G->base) fail(rescclInternalError, "group sequence underflow");
  while (G->pending.size() <= seq - G->base) G->pending.emplace_back();
  Pending& p = G->pending[seq - G->base];
  if (p.arrived == 0) {
    p.coll = coll;
    p.count = count;
    p.dtype = (int)dt;
    p.op = (int)op;
    p.algo = algo->s.get();
    p.send.assign(G->nranks, nullptr);
    p.recv.assign(G->nranks, nullptr);
  } else if (p.coll != coll || p.count != count || p.dtype != (int)dt || p.op != (int)op ||
             p.algo != algo->s.get()) {
    G->issued[comm->rank]--;
    fail(rescclInvalidUsage, "virtual ranks issued mismatching collectives");
  }
  p.send[comm->rank] = send;
  p.recv[comm->rank] = recv;
  p.streams.push_back(s);
  p.host |= host;
  p.arrived++;
  while (!G->pending.empty() && G->pending.front().arrived == G->nranks) {
    Pending q = G->pending.front();
    G->pending.pop_front();
    G->base++;
    if (q.count > 0) {
      if (q.host)
        group_host_launch(G, q);
      else
        group_launch(G, q);
    }
  }
}

// device-side epochs {mb_base, epoch, CTAs done}, zeroed (freed with the communicator)
unsigned long long* alloc_epochs(int dev) {
  cuda_check(cudaSetDevice(dev), "cudaSetDevice");
  unsigned long long* p = nullptr;
  cuda_check(cudaMalloc((void**)&p, 4 * sizeof(unsigned long long)), "cudaMalloc(epochs)");
  cuda_check(cudaMemset(p, 0, 4 * sizeof(unsigned long long)), "cudaMemset(epochs)");
  cuda_check(cudaDeviceSynchronize(), "cudaDeviceSynchronize");
  return p;
}

// ---------------------------------------------------------------- algorithm loading
rescclAlgo* load_algo(rescclComm* comm, const std::string& text) {
  std::shared_ptr<AlgoShared> s;
  if (comm->mode == 1) {
    Group* G = comm->group;
    auto it = G->algos.find(text);
    if (it != G->algos.end()) {
      s = it->second;
    } else {
      s = build_algo(text, comm->nranks);
      cuda_check(cudaSetDevice(G->dev), "cudaSetDevice");
      size_t bytes = (size_t)s->lay.region_bytes * G->nranks;
      cuda_check(cudaMalloc((void**)&s->region_alloc, bytes), "cudaMalloc(region)");
      cuda_check(cudaMemset(s->region_alloc, 0, bytes), "cudaMemset(region)");
      cuda_check(cudaDeviceSynchronize(), "cudaDeviceSynchronize");
      for (int q = 0; q < G->nranks; ++q) s->region.push_back(s->region_alloc + (size_t)q * s->lay.region_bytes);
      s->dev_epochs = alloc_epochs(G->dev);
      G->algos[text] = s;
    }
  } else {
    s = build_algo(text, comm->nranks);
    if (s->opt.direct) {
      if (comm->mode != 0)
        fail(rescclInvalidUsage, "direct=1 is supported for virtual ranks and multi-process communicators");
      s->twin = build_algo(text, comm->nranks, "direct=0");  // staged plan for unregistered buffers
    }
    for (AlgoShared* x : {s.get(), s->twin.get()}) {
      if (!x) continue;
      size_t need = (size_t)x->lay.region_bytes;
      if (comm->arena_used + need > comm->arena_bytes)
        fail(rescclInvalidUsage, "FIFO arena exhausted: need " + std::to_string(comm->arena_used + need) +
                                     " bytes; raise RESCCL_ARENA_BYTES");
      x->region_off = (int64_t)comm->arena_used;
      comm->arena_used += (need + 4095) / 4096 * 4096;
    }
  }
  auto algo = std::make_unique<rescclAlgo>();
  algo->s = s;
  algo->comm = comm;
  if (comm->mode != 1) {  // this rank's device-side epochs for the plan and its staged twin
    algo->dev_epochs[0] = alloc_epochs(comm->dev);
    if (s->twin) algo->dev_epochs[1] = alloc_epochs(comm->dev);
  }
  rescclAlgo* raw = algo.get();
  comm->algos.push_back(std::move(algo));
  comm->active[(int)s->ir.coll] = raw;
  comm->ranked[(int)s->ir.coll].push_back(raw);
  return raw;
}

rescclAlgo* ensure_algo(rescclComm* comm, Coll coll) {
  rescclAlgo* a = comm->active[(int)coll];
  if (a) return a;
  Ir ir = gen_ring(coll, comm->nranks);
  return load_algo(comm, ir.to_text());
}

// the algorithm a call of `bytes` (per-rank buffer S) runs: the most recently loaded or
// activated one of its collective whose [minbytes, maxbytes] holds it; else the active one
rescclAlgo* select_algo(rescclComm* comm, Coll coll, long long bytes) {
  const auto& v = comm->ranked[(int)coll];
  for (auto it = v.rbegin(); it != v.rend(); ++it) {
    const Options& o = (*it)->s->opt;
    if (bytes >= o.min_bytes && (o.max_bytes < 0 || bytes <= o.max_bytes)) return *it;
  }
  return ensure_algo(comm, coll);
}

Group* make_group(int dev, int n) {
  Group* G = new Group();
  G->dev = dev;
  G->nranks = n;
  G->issued.assign(n, 0);
  cuda_check(cudaSetDevice(dev), "cudaSetDevice");
  alloc_err_word(&G->err_host, &G->err_dev);
  return G;
}

Plan plan_from(const char* irText, const char* opts, Options* o_out, Ir* ir_out) {
  if (!irText) fail(rescclInvalidArgument, "irText is NULL");
  Ir ir = parse_any(irText);
  Options o = make_options(ir, opts);
  Plan p = make_plan(ir, o);
  if (o_out) *o_out = o;
  if (ir_out) *ir_out = ir;
  return p;
}


// ---------------------------------------------------------------- f3: NVLS windows and transport
// SURVEY §8(f) f3 (not in the paper): the NVSwitch-SHARP variant of the transport.  An
// NVLS window is device memory of every rank bound into one multicast object; calls of
// an algorithm loaded with nvls=1 whose buffers lie in NVLS windows run the NVLS kernel
// (rdev::nvls_run: mred / mcast on the collective's chunk layout), every other call runs
// the algorithm's primitive plan.  Driver entry points are resolved on first use so a
// driver without multicast only fails the NVLS calls.
constexpr size_t kNvlsHdr = 4096;  // barrier words [entry, exit] at the window's start

struct NvlsDriver {
  CUresult (*McCreate)(CUmemGenericAllocationHandle*, const CUmulticastObjectProp*) = nullptr;
  CUresult (*McAddDevice)(CUmemGenericAllocationHandle, CUdevice) = nullptr;
  CUresult (*McBindMem)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t, size_t,
                        unsigned long long) = nullptr;
  CUresult (*McUnbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t) = nullptr;
  CUresult (*McGetGranularity)(size_t*, const CUmulticastObjectProp*, CUmulticastGranularity_flags) = nullptr;
  CUresult (*MemCreate)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*, unsigned long long) =
      nullptr;
  CUresult (*MemRelease)(CUmemGenericAllocationHandle) = nullptr;
  CUresult (*MemAddressReserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long) = nullptr;
  CUresult (*MemAddressFree)(CUdeviceptr, size_t) = nullptr;
  CUresult (*MemMap)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long) = nullptr;
  CUresult (*MemUnmap)(CUdeviceptr, size_t) = nullptr;
  CUresult (*MemSetAccess)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t) = nullptr;
  CUresult (*MemExport)(void*, CUmemGenericAllocationHandle, CUmemAllocationHandleType, unsigned long long) =
      nullptr;
  CUresult (*MemImport)(CUmemGenericAllocationHandle*, void*, CUmemAllocationHandleType) = nullptr;
  CUresult (*DeviceGet)(CUdevice*, int) = nullptr;
  CUresult (*DeviceGetAttribute)(int*, CUdevice_attribute, CUdevice) = nullptr;
};

NvlsDriver& nvls_driver() {
  static NvlsDriver d;
  static bool ok = false;
  if (!ok) {
    driver();  // the base entry points first (fails cleanly without a driver)
    entry("cuMulticastCreate", &d.McCreate);
    entry("cuMulticastAddDevice", &d.McAddDevice);
    entry("cuMulticastBindMem", &d.McBindMem);
    entry("cuMulticastUnbind", &d.McUnbind);
    entry("cuMulticastGetGranularity", &d.McGetGranularity);
    entry("cuMemCreate", &d.MemCreate);
    entry("cuMemRelease", &d.MemRelease);
    entry("cuMemAddressReserve", &d.MemAddressReserve);
    entry("cuMemAddressFree", &d.MemAddressFree);
    entry("cuMemMap", &d.MemMap);
    entry("cuMemUnmap", &d.MemUnmap);
    entry("cuMemSetAccess", &d.MemSetAccess);
    entry("cuMemExportToShareableHandle", &d.MemExport);
    entry("cuMemImportFromShareableHandle", &d.MemImport);
    entry("cuDeviceGet", &d.DeviceGet);
    entry("cuDeviceGetAttribute", &d.DeviceGetAttribute);
    ok = true;
  }
  return d;
}

// one multicast object; released when the last window bound to it is released
struct McObj {
  CUmemGenericAllocationHandle h = 0;
  ~McObj() {
    if (h) nvls_driver().MemRelease(h);
  }
};

struct NvlsWin {
  std::shared_ptr<McObj> mc_obj;
  int dev = 0;
  size_t bytes = 0, total = 0;  // user bytes; mapped bytes (header + user, granularity-rounded)
  CUmemGenericAllocationHandle mc = 0, mem = 0;
  CUdeviceptr uc = 0, mcva = 0;
  bool added = false, bound = false, uc_mapped = false, mc_mapped = false;
  unsigned arrivals = 0;  // barrier arrivals per word after the calls issued so far
  char* user() const { return (char*)uc + kNvlsHdr; }
  char* user_mc() const { return (char*)mcva + kNvlsHdr; }
};

CUmulticastObjectProp nvls_prop(int nranks, size_t total, bool fabric) {
  CUmulticastObjectProp p;
  memset(&p, 0, sizeof(p));
  p.numDevices = (unsigned)nranks;
  p.size = total;
  p.handleTypes = fabric ? CU_MEM_HANDLE_TYPE_FABRIC : CU_MEM_HANDLE_TYPE_NONE;
  return p;
}

size_t nvls_total(int nranks, size_t bytes, bool fabric) {
  CUmulticastObjectProp p = nvls_prop(nranks, kNvlsHdr + bytes, fabric);
  size_t g = 0;
  cu_check(nvls_driver().McGetGranularity(&g, &p, CU_MULTICAST_GRANULARITY_RECOMMENDED),
           "cuMulticastGetGranularity");
  if (g == 0) g = 2 << 20;
  return (kNvlsHdr + bytes + g - 1) / g * g;
}

void nvls_add_device(NvlsWin& w) {
  CUdevice d;
  cu_check(nvls_driver().DeviceGet(&d, w.dev), "cuDeviceGet");
  cu_check(nvls_driver().McAddDevice(w.mc, d), "cuMulticastAddDevice");
  w.added = true;
}

// after every rank's device is added: this rank's memory, bound and mapped twice
void nvls_bind_map(NvlsWin& w) {
  NvlsDriver& D = nvls_driver();
  cuda_check(cudaSetDevice(w.dev), "cudaSetDevice");
  CUmemAllocationProp ap;
  memset(&ap, 0, sizeof(ap));
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = w.dev;
  cu_check(D.MemCreate(&w.mem, w.total, &ap, 0), "cuMemCreate");
  cu_check(D.McBindMem(w.mc, 0, w.mem, 0, w.total, 0), "cuMulticastBindMem");
  w.bound = true;
  CUmemAccessDesc ad;
  memset(&ad, 0, sizeof(ad));
  ad.location = ap.location;
  ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  cu_check(D.MemAddressReserve(&w.uc, w.total, 2 << 20, 0, 0), "cuMemAddressReserve");
  cu_check(D.MemMap(w.uc, w.total, 0, w.mem, 0), "cuMemMap(unicast)");
  w.uc_mapped = true;
  cu_check(D.MemSetAccess(w.uc, w.total, &ad, 1), "cuMemSetAccess(unicast)");
  cu_check(D.MemAddressReserve(&w.mcva, w.total, 2 << 20, 0, 0), "cuMemAddressReserve");
  cu_check(D.MemMap(w.mcva, w.total, 0, w.mc, 0), "cuMemMap(multicast)");
  w.mc_mapped = true;
  cu_check(D.MemSetAccess(w.mcva, w.total, &ad, 1), "cuMemSetAccess(multicast)");
  cuda_check(cudaMemset((void*)w.uc, 0, kNvlsHdr), "cudaMemset(nvls header)");
  cuda_check(cudaDeviceSynchronize(), "cudaDeviceSynchronize");
}

// best effort: every step that was taken is undone
void nvls_release(NvlsWin& w) {
  NvlsDriver& D = nvls_driver();
  cudaSetDevice(w.dev);
  cudaDeviceSynchronize();
  if (w.mc_mapped) D.MemUnmap(w.mcva, w.total);
  if (w.mcva) D.MemAddressFree(w.mcva, w.total);
  if (w.uc_mapped) D.MemUnmap(w.uc, w.total);
  if (w.uc) D.MemAddressFree(w.uc, w.total);
  if (w.bound) {
    CUdevice d;
    if (D.DeviceGet(&d, w.dev) == CUDA_SUCCESS) D.McUnbind(w.mc, d, 0, w.total);
  }
  if (w.mem) D.MemRelease(w.mem);
  w = NvlsWin();  // drops this window's reference to the multicast object
}

// the NVLS window of `comm` holding [p, p + bytes), or null
NvlsWin* nvls_find(rescclComm* comm, const void* p, size_t bytes) {
  for (auto& w : comm->nvls)
    if ((const char*)p >= w->user() && (const char*)p + bytes <= w->user() + w->bytes) return w.get();
  return nullptr;
}

std::string nvls_source(int coll) {
  return "#include \"resccl_device.cuh\"\n"
         "extern \"C\" __global__ void __launch_bounds__(512, 1) resccl_nvls_kernel(rdev::NvlsArgs a) {\n"
         "  rdev::nvls_run<RESCCL_T, RESCCL_OP, " +
         std::to_string(coll) + ">(a);\n}\n";
}

Kern& nvls_kernel(int dev, int coll, rescclDataType_t dt, rescclRedOp_t op) {
  static std::map<std::string, Kern> cache;  // per device (modules are per context)
  std::string key = std::to_string(dev) + "/" + std::to_string(coll) + "/" + std::to_string((int)dt) + "/" +
                    std::to_string((int)op);
  auto it = cache.find(key);
  if (it != cache.end()) return it->second;
  std::vector<char> cubin = nvrtc_compile(nvls_source(coll), dt, op, false);
  Kern k;
  cu_check(driver().ModuleLoadData(&k.mod, cubin.data()), "cuModuleLoadData(nvls)");
  cu_check(driver().ModuleGetFunction(&k.fn, k.mod, "resccl_nvls_kernel"), "cuModuleGetFunction(nvls)");
  return cache[key] = k;
}

struct NvlsArgsHost {  // mirrors rdev::NvlsArgs
  char* mc_send;
  char* mc_recv;
  const char* uc_send;
  char* uc_recv;
  unsigned* mc_flags;
  unsigned* uc_flags;
  long long lo_bytes, hi_bytes;
  unsigned target;
  int nranks;
  int vec;
  int* err;
  unsigned long long timeout_ns;
};

// NVLS eligibility of a call (rank-independent, so every rank decides alike) and launch.
// Returns false -- the caller runs the primitive plan -- when a buffer is outside the NVLS
// windows or at an offset that is not 4-byte aligned, a per-rank block is not whole
// 4-byte granules, or the op has no multimem form (f32 max/min).
bool try_nvls(rescclComm* comm, const AlgoShared& a, int coll, const void* send, void* recv, size_t count,
              rescclDataType_t dt, rescclRedOp_t op, cudaStream_t s) {
  if (comm->nvls.empty() || comm->mode == 1) return false;
  if (dt == rescclFloat32 && op != rescclSum) return false;
  const int N = comm->nranks, r = comm->rank;
  const long long e = elt_size(dt);
  const long long blk = (long long)count * e;  // AR: whole buffer; RS/AG: one rank's block
  const long long sbytes = coll == (int)Coll::ReduceScatter ? blk * N : blk;
  const long long rbytes = coll == (int)Coll::AllGather ? blk * N : blk;
  if (blk % 4) return false;
  // every buffer in an NVLS window (also RS's receive and AG's send buffer, which are
  // only touched locally): windows are symmetric, so the decision below is the same on
  // every rank
  NvlsWin* ws = nvls_find(comm, send, (size_t)sbytes);
  NvlsWin* wr = nvls_find(comm, recv, (size_t)rbytes);
  if (!ws || !wr) return false;
  const long long os = (const char*)send - ws->user();
  const long long orr = (char*)recv - wr->user();
  if (os % 4 || orr % 4) return false;
  NvlsWin& W = coll == (int)Coll::ReduceScatter ? *ws : *wr;  // carries the barrier words
  NvlsArgsHost ka;
  memset(&ka, 0, sizeof(ka));
  ka.mc_send = ws->user_mc() + os;
  ka.mc_recv = wr->user_mc() + orr;
  ka.uc_send = (const char*)send;
  ka.uc_recv = (char*)recv;
  ka.mc_flags = (unsigned*)W.mcva;
  ka.uc_flags = (unsigned*)W.uc;
  long long span;  // largest per-rank range (rank-independent grid)
  if (coll == (int)Coll::AllReduce) {
    // AR partition: 16-byte-aligned slices of ceil(S/N) (reading R28); any partition gives
    // the same result, each element is reduced by exactly one rank
    const long long sl = ((blk + N - 1) / N + 15) / 16 * 16;
    ka.lo_bytes = std::min(r * sl, blk);
    ka.hi_bytes = std::min(ka.lo_bytes + sl, blk);
    ka.vec = os % 16 == 0 && orr % 16 == 0;
    span = sl;
  } else {
    ka.lo_bytes = r * blk;
    ka.hi_bytes = ka.lo_bytes + blk;
    ka.vec = blk % 16 == 0 && os % 16 == 0 && orr % 16 == 0;
    span = blk;
  }
  const long long per_cta = 512LL * 4 * (ka.vec ? 16 : 4);
  const int grid = (int)std::max(1LL, std::min((long long)a.opt.nvls_ctas, (span + per_cta - 1) / per_cta));
  W.arrivals += (unsigned)(N * grid);
  ka.target = W.arrivals;
  ka.nranks = N;
  ka.err = comm->err_dev;
  ka.timeout_ns = timeout_ns();
  cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
  Kern& k = nvls_kernel(comm->dev, coll, dt, op);
  void* params[] = {&ka};
  cu_check(driver().LaunchCooperativeKernel(k.fn, grid, 1, 1, 512, 1, 1, 0, (CUstream)s, params),
           "cuLaunchCooperativeKernel(nvls)");
  return true;
}

// Multi-process NVLS window: rank 0 creates the multicast object and exports a fabric
// handle; every rank imports it, adds its device, then binds and maps its memory.  Every
// rank runs all three exchanges whatever happened locally, so a failure on any rank
// surfaces on every rank (same order of callback calls, no hang).
struct NvlsBlob {
  unsigned magic;
  int ok;
  unsigned long long total;
  CUmemFabricHandle handle;
  char msg[160];
};

void nvls_status(NvlsBlob& b, const std::string& m) {
  b.ok = 0;
  snprintf(b.msg, sizeof(b.msg), "%s", m.c_str());
}

void nvls_exchange(NvlsBlob& mine, std::vector<NvlsBlob>& all, int nranks,
                   int (*allgather)(const void*, void*, size_t, void*), void* ctx, const char* phase) {
  all.assign(nranks, NvlsBlob());
  if (allgather(&mine, all.data(), sizeof(NvlsBlob), ctx) != 0)
    fail(rescclSystemError, std::string("allgather callback failed (") + phase + ")");
  for (int q = 0; q < nranks; ++q) {
    if (all[q].magic != 0x4e564c53u) fail(rescclSystemError, std::string("corrupt NVLS blob (") + phase + ")");
    if (!all[q].ok)
      fail(rescclCudaError, std::string("NVLS window (") + phase + ") failed on rank " + std::to_string(q) + ": " +
                                std::string(all[q].msg, strnlen(all[q].msg, sizeof(all[q].msg))));
  }
}

}  // namespace

// =================================================================== C ABI
extern "C" {

const char* rescclGetErrorString(rescclResult_t r) {
  switch (r) {
    case rescclSuccess: return "success";
    case rescclInvalidArgument: return "invalid argument";
    case rescclInvalidUsage: return "invalid usage";
    case rescclCudaError: return "CUDA error";
    case rescclSystemError: return "system error";
    case rescclInternalError: return "internal error";
    case rescclTimeout: return "timeout (device watchdog)";
  }
  return "unknown result";
}

const char* rescclGetLastError(void) { return g_last_error.c_str(); }
int rescclGetVersion(void) { return RESCCL_VERSION; }

struct Blob {
  unsigned magic;
  int rank, nranks, dev;
  unsigned long long arena_bytes;
  cudaIpcMemHandle_t handle;
  int pid;
  unsigned long long host_piece;  // RESCCL_HOST_PIECE of this rank (must agree across ranks)
};

rescclResult_t rescclCommCreate(int rank, int nranks, int cudaDev, rescclComm_t* out) {
  API_BEGIN
  if (!out) fail(rescclInvalidArgument, "out is NULL");
  if (nranks < 1 || nranks > kMaxR || rank < 0 || rank >= nranks) fail(rescclInvalidArgument, "bad rank/nranks");
  auto c = std::make_unique<rescclComm>();
  c->rank = rank;
  c->nranks = nranks;
  c->dev = cudaDev;
  c->mode = 0;
  cuda_check(cudaSetDevice(cudaDev), "cudaSetDevice");
  c->arena_bytes = arena_default();
  c->host_piece = host_piece_bytes();
  cuda_check(cudaMalloc((void**)&c->arena, c->arena_bytes), "cudaMalloc(arena)");
  cuda_check(cudaMemset(c->arena, 0, c->arena_bytes), "cudaMemset(arena)");
  cuda_check(cudaDeviceSynchronize(), "cudaDeviceSynchronize");
  alloc_err_word(&c->err_host, &c->err_dev);
  c->peer_arena.assign(nranks, nullptr);
  c->peer_opened.assign(nranks, false);
  c->peer_arena[rank] = c->arena;
  *out = c.release();
  API_END
}

rescclResult_t rescclCommGetHandle(rescclComm_t comm, void* buf, size_t* len) {
  API_BEGIN
  if (!comm || !len) fail(rescclInvalidArgument, "null argument");
  if (comm->mode != 0) fail(rescclInvalidUsage, "handles exist only in multi-process mode");
  if (!buf) {
    *len = sizeof(Blob);
    return rescclSuccess;
  }
  if (*len < sizeof(Blob)) fail(rescclInvalidArgument, "handle buffer too small");
  Blob b;
  memset(&b, 0, sizeof(b));
  b.magic = 0x52435343u;
  b.rank = comm->rank;
  b.nranks = comm->nranks;
  b.dev = comm->dev;
  b.arena_bytes = comm->arena_bytes;
  b.pid = (int)getpid();
  b.host_piece = comm->host_piece;
  cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
  cuda_check(cudaIpcGetMemHandle(&b.handle, comm->arena), "cudaIpcGetMemHandle");
  memcpy(buf, &b, sizeof(b));
  *len = sizeof(Blob);
  API_END
}

rescclResult_t rescclCommConnect(rescclComm_t comm, const void* const* handles, const size_t* lens) {
  API_BEGIN
  if (!comm || !handles || !lens) fail(rescclInvalidArgument, "null argument");
  if (comm->mode != 0) fail(rescclInvalidUsage, "connect is for multi-process communicators");
  cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
  for (int q = 0; q < comm->nranks; ++q) {
    if (q == comm->rank) continue;
    if (!handles[q] || lens[q] < sizeof(Blob)) fail(rescclInvalidArgument, "bad handle blob");
    Blob b;
    memcpy(&b, handles[q], sizeof(b));
    if (b.magic != 0x52435343u || b.rank != q || b.nranks != comm->nranks)
      fail(rescclInvalidArgument, "handle blob of rank " + std::to_string(q) + " is inconsistent");
    if (b.arena_bytes != comm->arena_bytes) fail(rescclInvalidUsage, "ranks use different RESCCL_ARENA_BYTES");
    if (b.host_piece != comm->host_piece)
      fail(rescclInvalidUsage, "ranks use different RESCCL_HOST_PIECE (" + std::to_string(b.host_piece) + " on rank " +
                                   std::to_string(q) + ", " + std::to_string(comm->host_piece) + " here)");
    void* p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, b.handle, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess)
      fail(rescclSystemError, "cudaIpcOpenMemHandle(rank " + std::to_string(q) + "): " + cudaGetErrorString(e));
    comm->peer_arena[q] = (char*)p;
    comm->peer_opened[q] = true;
  }
  comm->connected = true;
  API_END
}

struct WinBlob {
  unsigned magic;
  int rank;
  unsigned long long bytes, offset;
  cudaIpcMemHandle_t handle;
};

rescclResult_t rescclCommRegister(rescclComm_t comm, void* ptr, size_t bytes, void* blob, size_t* len) {
  API_BEGIN
  if (!comm || !len) fail(rescclInvalidArgument, "null argument");
  if (comm->mode != 0) fail(rescclInvalidUsage, "windows are for multi-process communicators");
  if (!blob) {
    *len = sizeof(WinBlob);
    return rescclSuccess;
  }
  if (!ptr || bytes == 0) fail(rescclInvalidArgument, "null or empty window");
  if (*len < sizeof(WinBlob)) fail(rescclInvalidArgument, "blob buffer too small");
  cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
  CUdeviceptr base = 0;
  size_t asz = 0;
  cu_check(driver().MemGetAddressRange(&base, &asz, (CUdeviceptr)ptr), "cuMemGetAddressRange");
  if ((char*)ptr + bytes > (char*)base + asz) fail(rescclInvalidArgument, "window exceeds its allocation");
  WinBlob b;
  memset(&b, 0, sizeof(b));
  b.magic = 0x52574e44u;
  b.rank = comm->rank;
  b.bytes = bytes;
  b.offset = (char*)ptr - (char*)base;
  cuda_check(cudaIpcGetMemHandle(&b.handle, (void*)base), "cudaIpcGetMemHandle(window)");
  memcpy(blob, &b, sizeof(b));
  *len = sizeof(b);
  rescclComm::Window W;
  W.base = (char*)ptr;
  W.bytes = bytes;
  W.peer.assign(comm->nranks, nullptr);
  W.peer[comm->rank] = (char*)ptr;
  comm->windows.push_back(W);  // connected by rescclCommRegisterConnect
  API_END
}

rescclResult_t rescclCommRegisterConnect(rescclComm_t comm, const void* const* blobs, const size_t* lens,
                                         int* window) {
  API_BEGIN
  if (!comm || !blobs || !lens) fail(rescclInvalidArgument, "null argument");
  if (comm->windows.empty()) fail(rescclInvalidUsage, "rescclCommRegister first");
  auto& W = comm->windows.back();
  cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
  for (int q = 0; q < comm->nranks; ++q) {
    if (q == comm->rank) continue;
    if (!blobs[q] || lens[q] < sizeof(WinBlob)) fail(rescclInvalidArgument, "bad window blob");
    WinBlob b;
    memcpy(&b, blobs[q], sizeof(b));
    if (b.magic != 0x52574e44u || b.rank != q) fail(rescclInvalidArgument, "inconsistent window blob");
    if (b.bytes != W.bytes) fail(rescclInvalidUsage, "windows must have the same size on every rank");
    std::string key(reinterpret_cast<const char*>(&b.handle), sizeof(b.handle));
    key += "/" + std::to_string(q);
    auto it = comm->ipc_maps.find(key);
    char* mapped;
    if (it != comm->ipc_maps.end()) {
      mapped = it->second;
    } else {
      void* p = nullptr;
      cudaError_t e = cudaIpcOpenMemHandle(&p, b.handle, cudaIpcMemLazyEnablePeerAccess);
      if (e != cudaSuccess)
        fail(rescclSystemError, "cudaIpcOpenMemHandle(window of rank " + std::to_string(q) + "): " +
                                    cudaGetErrorString(e));
      mapped = (char*)p;
      comm->ipc_maps[key] = mapped;
    }
    W.peer[q] = mapped + b.offset;
  }
  if (window) *window = (int)comm->windows.size() - 1;
  API_END
}

rescclResult_t rescclCommInit(rescclComm_t* out, int rank, int nranks, int cudaDev,
                              int (*allgather)(const void*, void*, size_t, void*), void* ctx) {
  API_BEGIN
  if (!out || !allgather) fail(rescclInvalidArgument, "null argument");
  rescclComm_t c = nullptr;
  rescclResult_t r = rescclCommCreate(rank, nranks, cudaDev, &c);
  if (r != rescclSuccess) return r;
  std::vector<char> mine(sizeof(Blob)), all(sizeof(Blob) * nranks);
  size_t len = mine.size();
  r = rescclCommGetHandle(c, mine.data(), &len);
  if (r != rescclSuccess) {
    rescclCommDestroy(c);
    return r;
  }
  if (allgather(mine.data(), all.data(), sizeof(Blob), ctx) != 0) {
    rescclCommDestroy(c);
    fail(rescclSystemError, "allgather callback failed");
  }
  std::vector<const void*> hs(nranks);
  std::vector<size_t> ls(nranks, sizeof(Blob));
  for (int q = 0; q < nranks; ++q) hs[q] = all.data() + q * sizeof(Blob);
  r = rescclCommConnect(c, hs.data(), ls.data());
  if (r != rescclSuccess) {
    rescclCommDestroy(c);
    return r;
  }
  *out = c;
  API_END
}

rescclResult_t rescclCommInitAll(rescclComm_t* comms, int ndev, const int* devlist) {
  API_BEGIN
  if (!comms || ndev < 1 || ndev > kMaxR) fail(rescclInvalidArgument, "bad arguments");
  std::vector<int> devs(ndev, 0);
  if (devlist)
    for (int i = 0; i < ndev; ++i) devs[i] = devlist[i];
  bool all_same = true;
  for (int i = 1; i < ndev; ++i) all_same &= devs[i] == devs[0];
  bool all_distinct = true;
  for (int i = 0; i < ndev; ++i)
    for (int j = i + 1; j < ndev; ++j) all_distinct &= devs[i] != devs[j];
  if (!all_same && !all_distinct)
    fail(rescclInvalidUsage, "devlist must be one device repeated (virtual ranks) or distinct devices");
  std::vector<rescclComm*> cs;
  if (all_same && ndev > 1) {
    Group* G = make_group(devs[0], ndev);
    for (int r = 0; r < ndev; ++r) {
      auto c = new rescclComm();
      c->rank = r;
      c->nranks = ndev;
      c->dev = devs[0];
      c->mode = 1;
      c->host_piece = host_piece_bytes();
      c->group = G;
      c->connected = true;
      c->err_host = G->err_host;
      c->err_dev = G->err_dev;
      G->comms.push_back(c);
      G->refs++;
      cs.push_back(c);
    }
  } else {
    // distinct devices in one process (or a single rank): peer access + direct pointers
    for (int r = 0; r < ndev; ++r) {
      auto c = new rescclComm();
      c->rank = r;
      c->nranks = ndev;
      c->dev = devs[r];
      c->mode = 2;
      c->host_piece = host_piece_bytes();
      cuda_check(cudaSetDevice(devs[r]), "cudaSetDevice");
      for (int q = 0; q < ndev; ++q) {
        if (q == r) continue;
        cudaError_t e = cudaDeviceEnablePeerAccess(devs[q], 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
          fail(rescclCudaError, std::string("cudaDeviceEnablePeerAccess: ") + cudaGetErrorString(e));
        cudaGetLastError();
      }
      c->arena_bytes = arena_default();
      cuda_check(cudaMalloc((void**)&c->arena, c->arena_bytes), "cudaMalloc(arena)");
      cuda_check(cudaMemset(c->arena, 0, c->arena_bytes), "cudaMemset(arena)");
      alloc_err_word(&c->err_host, &c->err_dev);
      cs.push_back(c);
    }
    for (auto c : cs) {
      c->peer_arena.resize(ndev);
      for (int q = 0; q < ndev; ++q) c->peer_arena[q] = cs[q]->arena;
      c->peer_opened.assign(ndev, false);
      c->connected = true;
      c->peers_local = cs;
      cuda_check(cudaSetDevice(c->dev), "cudaSetDevice");
      cuda_check(cudaDeviceSynchronize(), "cudaDeviceSynchronize");
    }
  }
  for (int r = 0; r < ndev; ++r) comms[r] = cs[r];
  API_END
}

rescclResult_t rescclCommDestroy(rescclComm_t comm) {
  API_BEGIN
  if (!comm) return rescclSuccess;
  cudaSetDevice(comm->dev);
  cudaDeviceSynchronize();
  for (auto& w : comm->nvls) nvls_release(*w);
  comm->nvls.clear();
  if (comm->mode == 1) {
    Group* G = comm->group;
    if (--G->refs == 0) {
      for (auto& kv : G->algos) {
        for (auto& k : kv.second->kernels)
          if (k.second.mod) driver().ModuleUnload(k.second.mod);
        kv.second->kernels.clear();
        if (kv.second->region_alloc) cudaFree(kv.second->region_alloc);
        if (kv.second->dev_epochs) cudaFree(kv.second->dev_epochs);
        if (kv.second->phase_dev) cudaFree(kv.second->phase_dev);
        if (kv.second->trace_host) cudaFreeHost(kv.second->trace_host);
      }
      for (auto e : G->events) cudaEventDestroy(e);
      G->hcopy.release();
      cudaFreeHost(G->err_host);
      delete G;
    }
    // this rank's buffers (the group's other comms may already be deleted)
    if (comm->scratch) cudaFree(comm->scratch);
    for (char* q : comm->retired_scratch) cudaFree(q);
    if (comm->hstage) cudaFree(comm->hstage);
  } else {
    for (auto& a : comm->algos) {
      for (auto* e : a->dev_epochs)
        if (e) cudaFree(e);
      if (a->s.use_count() == 1)
        for (AlgoShared* x : {a->s.get(), a->s->twin.get()})
          if (x) {
            for (auto& k : x->kernels)
              if (k.second.mod) driver().ModuleUnload(k.second.mod);
            if (x->phase_dev) cudaFree(x->phase_dev);
            if (x->trace_host) cudaFreeHost(x->trace_host);
          }
    }
    for (int q = 0; q < (int)comm->peer_opened.size(); ++q)
      if (comm->peer_opened[q]) cudaIpcCloseMemHandle(comm->peer_arena[q]);
    for (auto& kv : comm->ipc_maps) cudaIpcCloseMemHandle(kv.second);
    if (comm->arena) cudaFree(comm->arena);
    if (comm->err_host) cudaFreeHost(comm->err_host);
    if (comm->scratch) cudaFree(comm->scratch);
    for (char* q : comm->retired_scratch) cudaFree(q);
    if (comm->hstage) cudaFree(comm->hstage);
    comm->hcopy.release();
  }
  delete comm;
  API_END
}

rescclResult_t rescclCommRank(rescclComm_t comm, int* rank) {
  API_BEGIN
  if (!comm || !rank) fail(rescclInvalidArgument, "null argument");
  *rank = comm->rank;
  API_END
}

rescclResult_t rescclCommCount(rescclComm_t comm, int* nranks) {
  API_BEGIN
  if (!comm || !nranks) fail(rescclInvalidArgument, "null argument");
  *nranks = comm->nranks;
  API_END
}

rescclResult_t rescclCommCuDevice(rescclComm_t comm, int* device) {
  API_BEGIN
  if (!comm || !device) fail(rescclInvalidArgument, "null argument");
  *device = comm->dev;
  API_END
}

rescclResult_t rescclCommGetAsyncError(rescclComm_t comm, rescclResult_t* err) {
  API_BEGIN
  if (!comm || !err) fail(rescclInvalidArgument, "null argument");
  volatile int* w = comm->err_host;
  *err = (w && *w) ? rescclTimeout : rescclSuccess;
  API_END
}

rescclResult_t rescclLoadAlgorithm(rescclComm_t comm, const char* irText, rescclAlgo_t* out) {
  API_BEGIN
  if (!comm || !irText) fail(rescclInvalidArgument, "null argument");
  if (!comm->connected) fail(rescclInvalidUsage, "communicator not connected");
  rescclAlgo* a = load_algo(comm, irText);
  if (out) *out = a;
  API_END
}

rescclResult_t rescclSetActiveAlgorithm(rescclComm_t comm, rescclAlgo_t algo) {
  API_BEGIN
  if (!comm || !algo || algo->comm != comm) fail(rescclInvalidArgument, "algorithm does not belong to comm");
  comm->active[(int)algo->s->ir.coll] = algo;
  auto& v = comm->ranked[(int)algo->s->ir.coll];
  v.erase(std::remove(v.begin(), v.end(), algo), v.end());
  v.push_back(algo);
  API_END
}

rescclResult_t rescclGetPlanInfo(rescclAlgo_t algo, char* json, size_t* len) {
  API_BEGIN
  if (!algo) fail(rescclInvalidArgument, "algo is NULL");
  if (algo->s->json.empty()) algo->s->json = info_json(*algo->s);
  write_out(algo->s->json, json, len);
  API_END
}

rescclResult_t rescclGetPhaseTrace(rescclAlgo_t algo, void* buf, size_t* len) {
  API_BEGIN
  if (!algo) fail(rescclInvalidArgument, "algo is NULL");
  if (!len) fail(rescclInvalidArgument, "len is NULL");
  AlgoShared& a = *algo->s;
  if (!a.opt.phase || !a.phase_dev) fail(rescclInvalidUsage, "no phase trace: load with phase=1 and run");
  const size_t per = (size_t)RESCCL_PH_MAX_HOST * 8;
  const size_t words = 4 + (size_t)a.phase_blocks * 2 * per;
  if (!buf) {
    *len = words * sizeof(unsigned long long);
    return rescclSuccess;
  }
  if (*len < words * sizeof(unsigned long long)) {
    *len = words * sizeof(unsigned long long);
    fail(rescclInvalidArgument, "buffer too small");
  }
  auto* out = (unsigned long long*)buf;
  out[0] = (unsigned long long)a.phase_blocks;
  out[1] = (unsigned long long)a.phase_block_base;
  out[2] = (unsigned long long)RESCCL_PH_MAX_HOST;
  out[3] = (unsigned long long)a.opt.instances;
  cuda_check(cudaSetDevice(a.phase_dev_id), "cudaSetDevice");
  cuda_check(cudaDeviceSynchronize(), "cudaDeviceSynchronize");
  cuda_check(cudaMemcpy(out + 4, a.phase_dev, (words - 4) * sizeof(unsigned long long), cudaMemcpyDeviceToHost),
             "cudaMemcpy(phase)");
  *len = words * sizeof(unsigned long long);
  API_END
}

rescclResult_t rescclGetTbUtilization(rescclAlgo_t algo, char* json, size_t* len) {
  API_BEGIN
  if (!algo) fail(rescclInvalidArgument, "algo is NULL");
  AlgoShared& a = *algo->s;
  if (!a.opt.trace || !a.trace_host) fail(rescclInvalidUsage, "no trace: load with trace=1 (RESCCL_TRACE=1) and run");
  std::ostringstream o;
  o << "{\"lanes\":[";
  double sum_idle = 0, max_idle = 0, csum = 0, cmax = 0;
  int n = 0, nc = 0;
  unsigned long long t_min = ~0ull, t_max = 0;
  bool first = true;
  for (int b = 0; b < a.trace_blocks; ++b) {
    int g = b + a.trace_block_base;
    int pair = g / a.opt.instances, inst = g % a.opt.instances;
    int rank = 0;
    while (rank + 1 < (int)a.lay.pair_start.size() && a.lay.pair_start[rank + 1] <= pair) ++rank;
    int cta = pair - a.lay.pair_start[rank];
    unsigned long long cb = ~0ull, ce = 0;
    for (int lane = 0; lane < 2; ++lane) {
      volatile unsigned long long* tr = a.trace_host + 8 * (2 * (size_t)b + lane);
      if (tr[1] <= tr[0]) continue;
      cb = std::min(cb, (unsigned long long)tr[0]);
      ce = std::max(ce, (unsigned long long)tr[1]);
      if (tr[3] == 0) continue;
      double life = (double)(tr[1] - tr[0]);
      double idle = (double)tr[2] / life;
      if (idle > 1) idle = 1;
      sum_idle += idle;
      max_idle = std::max(max_idle, idle);
      ++n;
      t_min = std::min(t_min, (unsigned long long)tr[0]);
      t_max = std::max(t_max, (unsigned long long)tr[1]);
      o << (first ? "" : ",") << "[" << rank << "," << cta << "," << inst << "," << lane << "," << (tr[1] - tr[0])
        << "," << tr[2] << "," << tr[3] << "]";
      first = false;
    }
    if (ce > cb) {  // the CTA (one SM): both lanes busy-waiting or finished
      double ci = (double)a.trace_host[8 * (2 * (size_t)b) + 4] / (double)(ce - cb);
      if (ci > 1) ci = 1;
      csum += ci;
      cmax = std::max(cmax, ci);
      ++nc;
    }
  }
  double avg = n ? sum_idle / n : 0, cavg = nc ? csum / nc : 0;
  o << "],\"fields\":[\"rank\",\"cta\",\"instance\",\"lane\",\"lifetime_ns\",\"wait_ns\",\"prims\"]"
    << ",\"tbs\":" << n << ",\"comm_time\":" << (1 - avg) << ",\"avg_idle\":" << avg
    << ",\"max_idle\":" << max_idle << ",\"ctas\":" << nc << ",\"cta_comm_time\":" << (1 - cavg)
    << ",\"cta_avg_idle\":" << cavg << ",\"cta_max_idle\":" << cmax
    << ",\"span_ns\":" << (n ? t_max - t_min : 0) << "}";
  write_out(o.str(), json, len);
  API_END
}

rescclResult_t rescclAllReduce(const void* sendbuf, void* recvbuf, size_t count, rescclDataType_t dtype,
                               rescclRedOp_t op, rescclComm_t comm, void* stream) {
  API_BEGIN
  collective(comm, (int)Coll::AllReduce, sendbuf, recvbuf, count, dtype, op, stream);
  API_END
}

rescclResult_t rescclAllGather(const void* sendbuf, void* recvbuf, size_t sendcount, rescclDataType_t dtype,
                               rescclComm_t comm, void* stream) {
  API_BEGIN
  collective(comm, (int)Coll::AllGather, sendbuf, recvbuf, sendcount, dtype, rescclSum, stream);
  API_END
}

rescclResult_t rescclReduceScatter(const void* sendbuf, void* recvbuf, size_t recvcount, rescclDataType_t dtype,
                                   rescclRedOp_t op, rescclComm_t comm, void* stream) {
  API_BEGIN
  collective(comm, (int)Coll::ReduceScatter, sendbuf, recvbuf, recvcount, dtype, op, stream);
  API_END
}

// ------------------------------------------------------------------ host-only tools
// ---------------------------------------------------------------- f3: NVLS windows
rescclResult_t rescclNvlsSupported(rescclComm_t comm, int* supported) {
  API_BEGIN
  if (!comm || !supported) fail(rescclInvalidArgument, "null argument");
  *supported = 0;
  if (comm->mode == 1) return rescclSuccess;  // virtual ranks share one device
  NvlsDriver& D = nvls_driver();
  CUdevice d;
  cu_check(D.DeviceGet(&d, comm->dev), "cuDeviceGet");
  int v = 0;
  cu_check(D.DeviceGetAttribute(&v, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, d), "cuDeviceGetAttribute");
  *supported = v;
  API_END
}

rescclResult_t rescclNvlsAlloc(rescclComm_t comm, size_t bytes, int (*allgather)(const void*, void*, size_t, void*),
                               void* ctx, void** ptr) {
  API_BEGIN
  if (!comm || !allgather || !ptr) fail(rescclInvalidArgument, "null argument");
  if (bytes == 0) fail(rescclInvalidArgument, "empty NVLS window");
  if (comm->mode != 0) fail(rescclInvalidUsage, "rescclNvlsAlloc is for multi-process communicators (see rescclNvlsAllocAll)");
  *ptr = nullptr;
  auto w = std::make_shared<NvlsWin>();
  w->dev = comm->dev;
  w->bytes = bytes;
  NvlsBlob mine;
  memset(&mine, 0, sizeof(mine));
  mine.magic = 0x4e564c53u;
  mine.ok = 1;
  std::vector<NvlsBlob> all;
  try {
    // 1: rank 0 creates and exports the multicast object; everyone agrees on its size
    try {
      cuda_check(cudaSetDevice(comm->dev), "cudaSetDevice");
      w->total = nvls_total(comm->nranks, bytes, true);
      mine.total = w->total;
      if (comm->rank == 0) {
        CUmulticastObjectProp p = nvls_prop(comm->nranks, w->total, true);
        cu_check(nvls_driver().McCreate(&w->mc, &p), "cuMulticastCreate");
        w->mc_obj = std::make_shared<McObj>();
        w->mc_obj->h = w->mc;
        cu_check(nvls_driver().MemExport(&mine.handle, w->mc, CU_MEM_HANDLE_TYPE_FABRIC, 0),
                 "cuMemExportToShareableHandle(fabric)");
      }
    } catch (Error& e) {
      nvls_status(mine, e.msg);
    }
    nvls_exchange(mine, all, comm->nranks, allgather, ctx, "create");
    for (auto& b : all)
      if (b.total != w->total) fail(rescclInvalidUsage, "NVLS windows must have the same size on every rank");
    // 2: import and add this rank's device
    try {
      if (comm->rank != 0) {
        cu_check(nvls_driver().MemImport(&w->mc, &all[0].handle, CU_MEM_HANDLE_TYPE_FABRIC),
                 "cuMemImportFromShareableHandle(fabric)");
        w->mc_obj = std::make_shared<McObj>();
        w->mc_obj->h = w->mc;
      }
      nvls_add_device(*w);
    } catch (Error& e) {
      nvls_status(mine, e.msg);
    }
    nvls_exchange(mine, all, comm->nranks, allgather, ctx, "add device");
    // 3: bind and map (every device is in the object now)
    try {
      nvls_bind_map(*w);
    } catch (Error& e) {
      nvls_status(mine, e.msg);
    }
    nvls_exchange(mine, all, comm->nranks, allgather, ctx, "bind");
  } catch (...) {
    nvls_release(*w);
    throw;
  }
  comm->nvls.push_back(w);
  *ptr = w->user();
  API_END
}

rescclResult_t rescclNvlsAllocAll(rescclComm_t* comms, int n, size_t bytes, void** ptrs) {
  API_BEGIN
  if (!comms || !ptrs || n < 1) fail(rescclInvalidArgument, "bad arguments");
  if (bytes == 0) fail(rescclInvalidArgument, "empty NVLS window");
  for (int k = 0; k < n; ++k) {
    if (!comms[k] || comms[k]->rank != k || comms[k]->nranks != n)
      fail(rescclInvalidArgument, "comms must be ranks 0..n-1 of one communicator");
    if (comms[k]->mode != 2) fail(rescclInvalidUsage, "rescclNvlsAllocAll needs one device per rank (rescclCommInitAll with distinct devices)");
  }
  std::vector<std::shared_ptr<NvlsWin>> ws(n);
  try {
    cuda_check(cudaSetDevice(comms[0]->dev), "cudaSetDevice");
    const size_t total = nvls_total(n, bytes, false);
    CUmulticastObjectProp p = nvls_prop(n, total, false);
    auto mco = std::make_shared<McObj>();
    cu_check(nvls_driver().McCreate(&mco->h, &p), "cuMulticastCreate");
    const CUmemGenericAllocationHandle mc = mco->h;
    for (int k = 0; k < n; ++k) {
      ws[k] = std::make_shared<NvlsWin>();
      ws[k]->mc_obj = mco;
      ws[k]->dev = comms[k]->dev;
      ws[k]->bytes = bytes;
      ws[k]->total = total;
      ws[k]->mc = mc;
    }
    for (int k = 0; k < n; ++k) nvls_add_device(*ws[k]);
    for (int k = 0; k < n; ++k) nvls_bind_map(*ws[k]);
  } catch (...) {
    for (int k = n - 1; k >= 0; --k)
      if (ws[k]) nvls_release(*ws[k]);
    throw;
  }
  for (int k = 0; k < n; ++k) {
    comms[k]->nvls.push_back(ws[k]);
    ptrs[k] = ws[k]->user();
  }
  API_END
}

rescclResult_t rescclNvlsFree(rescclComm_t comm, void* ptr) {
  API_BEGIN
  if (!comm || !ptr) fail(rescclInvalidArgument, "null argument");
  for (size_t i = 0; i < comm->nvls.size(); ++i)
    if (comm->nvls[i]->user() == (char*)ptr) {
      nvls_release(*comm->nvls[i]);
      comm->nvls.erase(comm->nvls.begin() + i);
      return rescclSuccess;
    }
  fail(rescclInvalidArgument, "not an NVLS window of this communicator");
  API_END
}

rescclResult_t rescclCompileNvls(rescclColl_t coll, rescclDataType_t dtype, rescclRedOp_t op, size_t* cubin_bytes) {
  API_BEGIN
  if (!cubin_bytes) fail(rescclInvalidArgument, "null argument");
  if ((int)coll < 0 || (int)coll > 2 || elt_size(dtype) == 0 || (int)op < 0 || (int)op > 2)
    fail(rescclInvalidArgument, "bad coll/dtype/op");
  *cubin_bytes = nvrtc_compile(nvls_source((int)coll), dtype, op, false).size();
  API_END
}

rescclResult_t rescclGenerateIr(const char* name, rescclColl_t coll, int nranks, const char* opts, char* text,
                                size_t* len) {
  API_BEGIN
  if (!name) fail(rescclInvalidArgument, "name is NULL");
  std::map<std::string, long> o;
  for (auto& kv : parse_kv(opts)) o[kv.first] = to_long(kv.second, kv.first);
  Ir ir = generate(name, (Coll)coll, nranks, o);
  write_out(ir.to_text(), text, len);
  API_END
}

rescclResult_t rescclProfilePlanner(const char* program, const char* opts, int verify, char* json, size_t* len) {
  API_BEGIN
  if (!program) fail(rescclInvalidArgument, "program is NULL");
  using clk = std::chrono::steady_clock;
  auto ms = [](clk::time_point a, clk::time_point b) {
    return std::chrono::duration<double, std::milli>(b - a).count();
  };
  auto t0 = clk::now();
  Ir ir = parse_any(program);                       // Parsing
  auto t1 = clk::now();
  Options o = make_options(ir, opts);
  Dag d = build_dag(ir);                            // Analysis
  auto t2 = clk::now();
  auto pr = o.sched ? round_robin(ir, d, o.model) : hpds(ir, d, o.model);  // Scheduling
  auto t3 = clk::now();
  Plan p = lower(ir, o.model, false, &pr, o.direct != 0, o.pushreduce != 0);  // Lowering (translation + TB allocation)
  Layout L = make_layout(p, o.fifo_depth, o.instances, o.chunk_bytes);
  CodegenOpts co = codegen_opts(o);
  co.rank_lo = 0;
  co.rank_hi = 1;
  std::string src = codegen(p, L, co);              // kernel source of rank 0
  auto t4 = clk::now();
  bool ok = true;
  if (verify) ok = deadlock_free(p, 1, 2);
  auto t5 = clk::now();
  int max_cta = 0;
  for (auto& r : p.ranks) max_cta = std::max(max_cta, (int)r.ctas.size());
  std::ostringstream out;
  out << "{\"nranks\":" << ir.nranks << ",\"tasks\":" << ir.t.size() << ",\"edges\":" << d.edges.size()
      << ",\"subpipelines\":" << pr.size() << ",\"max_ctas_per_rank\":" << max_cta
      << ",\"parse_ms\":" << ms(t0, t1) << ",\"analysis_ms\":" << ms(t1, t2) << ",\"schedule_ms\":" << ms(t2, t3)
      << ",\"lower_ms\":" << ms(t3, t4) << ",\"verify_ms\":" << ms(t4, t5)
      << ",\"deadlock_free\":" << (verify ? (ok ? "true" : "false") : "null")  // null: not checked
      << ",\"rank0_src_bytes\":" << src.size() << "}";
  write_out(out.str(), json, len);
  API_END
}

rescclResult_t rescclParseResCCLang(const char* program, char* irText, size_t* len) {
  API_BEGIN
  if (!program) fail(rescclInvalidArgument, "program is NULL");
  write_out(parse_rescclang(program).to_text(), irText, len);
  API_END
}

rescclResult_t rescclPlanIr(const char* irText, const char* opts, char* json, size_t* len) {
  API_BEGIN
  Options o;
  Plan p = plan_from(irText, opts, &o, nullptr);
  AlgoShared a;
  a.opt = o;
  a.plan = p;
  a.ir = p.ir;
  a.lay = make_layout(p, o.fifo_depth, o.instances, o.chunk_bytes);
  write_out(info_json(a), json, len);
  API_END
}

rescclResult_t rescclCodegenIr(const char* irText, const char* opts, int rank_lo, int rank_hi, char* src,
                               size_t* len) {
  API_BEGIN
  Options o;
  Plan p = plan_from(irText, opts, &o, nullptr);
  if (rank_lo < 0 || rank_hi > p.ir.nranks || rank_lo >= rank_hi) fail(rescclInvalidArgument, "bad rank range");
  Layout L = make_layout(p, o.fifo_depth, o.instances, o.chunk_bytes);
  CodegenOpts co = codegen_opts(o);
  co.rank_lo = rank_lo;
  co.rank_hi = rank_hi;
  write_out(codegen(p, L, co), src, len);
  API_END
}

rescclResult_t rescclCompileIr(const char* irText, const char* opts, rescclDataType_t dtype, rescclRedOp_t op,
                               size_t* cubin_bytes) {
  API_BEGIN
  Options o;
  Plan p = plan_from(irText, opts, &o, nullptr);
  Layout L = make_layout(p, o.fifo_depth, o.instances, o.chunk_bytes);
  CodegenOpts co = codegen_opts(o);
  co.rank_lo = 0;
  co.rank_hi = p.ir.nranks;
  co.gpu_scope = true;
  if (o.sys_rank >= 0) {  // one rank of a multi-process communicator
    if (o.sys_rank >= p.ir.nranks) fail(rescclInvalidArgument, "sysrank out of range");
    co.rank_lo = o.sys_rank;
    co.rank_hi = o.sys_rank + 1;
    co.gpu_scope = false;
    co.exit_barrier = o.direct;
  }
  auto cub = nvrtc_compile(codegen(p, L, co), dtype, op, co.gpu_scope);
  if (cubin_bytes) *cubin_bytes = cub.size();
  API_END
}

rescclResult_t rescclSimulateTimeline(const char* irText, const char* opts, const char* params, char* json,
                                      size_t* len) {
  API_BEGIN
  Options o;
  Plan p = plan_from(irText, opts, &o, nullptr);
  TimelineParams tp;
  long long count = 0;
  int elt = 2;
  for (auto& kv : parse_kv(params)) {
    double v;
    try {
      v = std::stod(kv.second);
    } catch (...) {
      fail(rescclInvalidArgument, "timeline parameter " + kv.first + " is not a number");
    }
    if (kv.first == "alpha") tp.alpha = v;
    else if (kv.first == "beta") tp.beta = v;
    else if (kv.first == "gamma") tp.gamma = v;
    else if (kv.first == "count") count = (long long)v;
    else if (kv.first == "elt") elt = (int)v;
    else fail(rescclInvalidArgument, "unknown timeline parameter " + kv.first);
  }
  if (count <= 0 || (elt != 2 && elt != 4)) fail(rescclInvalidArgument, "timeline needs count > 0 and elt 2|4");
  Geometry g = geometry(p.ir.coll, p.ir.nranks, count, elt, o.chunk_bytes, o.instances);
  tp.n_mb = g.n_mb;
  tp.c = (double)g.Mi * elt;
  tp.K = o.fifo_depth;
  tp.instances = o.instances;
  TimelineResult r = simulate_timeline(p, tp);
  write_out(timeline_json(p, tp, r), json, len);
  API_END
}

rescclResult_t rescclCheckDeadlock(const char* irText, const char* opts, int K, int n_mb, int* ok) {
  API_BEGIN
  if (!ok) fail(rescclInvalidArgument, "ok is NULL");
  Plan p = plan_from(irText, opts, nullptr, nullptr);
  *ok = deadlock_free(p, K, n_mb) ? 1 : 0;
  API_END
}

}  // extern "C"
