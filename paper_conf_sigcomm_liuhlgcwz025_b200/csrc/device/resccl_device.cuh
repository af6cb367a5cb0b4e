// ResCCL L0 transport device library for sm_100a.
//
// Compiled twice: by NVRTC together with the code the kernel generator emits for
// one schedule (csrc/plan/codegen.cc), and by nvcc in the build self-test.  It
// must therefore not include any system header.
//
// Execution model (§4.5): one generated kernel per
// schedule; block -> (rank, TB, instance); a TB is two independent warp groups
// ("lanes", reading R20): warps [0, W/2) run the send-lane primitive list and warps
// [W/2, W) the recv-lane list.  Each primitive loops over all micro-batches before
// the next one starts (task-level execution).  For micro-batch j a
// primitive
//   1. waits until every local dependency finished micro-batch j (rule (1)):
//      ld.acquire on a 64-bit monotone counter >= mb_base + j + 1;
//   2. waits for payload (recv) in its link FIFO slot and/or for FIFO credit (send):
//      ld.acquire on the slot flag / on the credit counter the receiver writes back;
//   3. moves 16-byte vectors (or elements on a misaligned tail): send, recv, rrc
//      (recvReduceCopy), rrs (recvReduceSend), rcs (recvCopySend), rrcs; bf16/fp16
//      combine in fp32 and round to nearest even on every store (reading R8);
//   4. publishes: fence, then the slot flag in the receiver's arena, the credit in
//      the sender's arena and the local completion counter.
// FIFOs live in the receiver's arena (one per link and instance, depth K, slot =
// one micro-batch slice); every 64-bit flag/counter is monotone across calls, so
// no reset kernel is needed.
#pragma once

#ifndef RESCCL_MAXR
#define RESCCL_MAXR 32
#endif
#ifndef RESCCL_TMA
#define RESCCL_TMA 1
#endif
#ifndef RESCCL_TRACE
#define RESCCL_TRACE 0
#endif
// RESCCL_PHASE: per-(primitive, micro-batch) %globaltimer phase records of every lane
// leader (device memory, read back by rescclGetPhaseTrace): where a hop's time goes
// (dependency wait, flag / credit wait, data movement, fence + post).
#ifndef RESCCL_PHASE
#define RESCCL_PHASE 0
#endif
#define RESCCL_PH_MAX 96   // records per (block, lane); record 0 = lane header

namespace rdev {

typedef unsigned long long u64;
typedef long long i64;
typedef unsigned int u32;
typedef unsigned short u16;

struct KArgs {
  char* arena[RESCCL_MAXR];           // plan region of every rank's arena (peer-mapped)
  const char* sendbuf[RESCCL_MAXR];   // per local rank (virtual mode: every rank)
  char* recvbuf[RESCCL_MAXR];
  char* scratch[RESCCL_MAXR];
  u64 mb_base;                        // micro-batches of this plan issued before this call
  i64 count;                          // AR: count; AG: sendcount; RS: recvcount (elements)
  i64 C;                              // algorithm-chunk elements
  i64 M;                              // micro-batch elements
  i64 Mi;                             // instance-slice elements
  int n_mb;
  int block_base;                     // global block id of blockIdx.x == 0
  int* err;                           // host-mapped error word
  u64 timeout_ns;
  u64* trace;                         // RESCCL_TRACE: 8 x u64 per (block, lane), host-mapped
  u64 epoch;                          // RESCCL_EXIT_BARRIER: calls of this plan issued before
  u64* epochs;                        // device-side epochs (graph-capturable launches), or null:
                                      // {mb_base, epoch, CTAs done}; the kernel reads the first two
                                      // instead of the fields above, the last CTA advances them
  u64* phase;                         // RESCCL_PHASE: RESCCL_PH_MAX x 8 u64 per (block, lane), or null
};

// CTA barrier that tolerates warp divergence (barrier.sync without .aligned): a lane's
// leader thread runs leader-only primitives (flag loops) while the rest of its warp has
// already moved on, so the block-wide barriers after the lanes' lists and the lane
// barriers may be reached by a warp's threads at different times (__syncthreads is the
// .aligned form, undefined under divergence; compute-sanitizer synccheck flags it)
__device__ __forceinline__ void cta_sync() { asm volatile("barrier.sync 0;" ::: "memory"); }

// Device-side epochs: every CTA takes this launch's micro-batch base and call epoch from
// device memory (so a CUDA graph replays with fresh epochs).  Each CTA reads them with
// acquire loads (its arrival below cannot overtake the reads) and then counts itself in;
// the LAST CTA to arrive -- every CTA of this launch has read the old values by then --
// advances them by this call's micro-batches / one call and resets the count, right at
// the start of the kernel, off its critical path (r02: the former end-of-kernel fence +
// atomic cost every launch ~1-2 us of tail).  Stream order makes the update visible to
// the next launch of the plan.
__device__ __forceinline__ const KArgs* epochs_begin(const KArgs& a, KArgs* sh) {
  if (!a.epochs) return &a;
  // thread 0 issues the two epoch loads first (their latency overlaps the copy); every
  // thread copies a slice of the kernel arguments into shared memory
  u64 v0 = 0, v1 = 0;
  if (threadIdx.x == 0) {
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v0) : "l"(&a.epochs[0]) : "memory");
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v1) : "l"(&a.epochs[1]) : "memory");
  }
  {
    const u64* src = (const u64*)&a;
    u64* dst = (u64*)sh;
    for (int i = threadIdx.x; i < (int)(sizeof(KArgs) / 8); i += blockDim.x) dst[i] = src[i];
  }
  cta_sync();
  if (threadIdx.x == 0) {
    sh->mb_base = v0;
    sh->epoch = v1;
  }
  cta_sync();
  // one thread of warp 1 counts this CTA in (its operand depends on the epoch values, so
  // the arrival cannot be performed before thread 0's loads returned -- they reached
  // shared memory before the barrier); the last CTA to arrive advances the epochs.  Warp
  // 0's leader starts its lane without waiting for the round trip.
  if (threadIdx.x == 32 || (blockDim.x <= 32 && threadIdx.x == 0)) {
    const u64 mb = sh->mb_base, ep = sh->epoch;
    u64 z;
    asm volatile("xor.b64 %0, %1, %1;" : "=l"(z) : "l"(mb ^ ep));
    const unsigned long long old = atomicAdd((unsigned long long*)&a.epochs[2], 1ull + z);
    if (old == (unsigned long long)gridDim.x - 1) {
      a.epochs[0] = mb + (u64)a.n_mb;
      a.epochs[1] = ep + 1;
      a.epochs[2] = 0;
    }
  }
  return sh;
}
__device__ __forceinline__ void epochs_end(const KArgs&) {}

enum : int { kRecv = 1, kSend = 2, kReduce = 4, kStore = 8, kCopy = 16, kDirect = 32, kPull = 64, kSendPull = 128 };
enum : int { BufNone = -1, BufSend = 0, BufRecv = 1, BufScratch = 2 };
enum : int { CollAllGather = 0, CollReduceScatter = 1, CollAllReduce = 2 };
enum : int { OpSum = 0, OpMax = 1, OpMin = 2 };
enum : int { kErrTimeout = 7 };

// ----------------------------------------------------------------------------- memory ops
#if defined(RESCCL_SCOPE_GPU)
#define RESCCL_SC ".gpu"
#else
#define RESCCL_SC ".sys"
#endif

__device__ __forceinline__ u64 ld_acquire_raw(const u64* p) {
  u64 v;
  asm volatile("ld.acquire" RESCCL_SC ".global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(u64* p, u64 v) {
  asm volatile("st.relaxed" RESCCL_SC ".global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
#ifndef RESCCL_JITTER
#define RESCCL_JITTER 0
#endif
// Fault injector (RESCCL_JITTER=1, debug): a pseudo-random 0..~8 us delay before every
// flag / credit / counter post and after every successful acquire, to shake out
// memory-ordering bugs (SURVEY §5 race detection).
__device__ __forceinline__ void jitter() {
#if RESCCL_JITTER
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  unsigned x = (unsigned)(t ^ (t >> 17)) * 2654435761u + (unsigned)clock() + threadIdx.x * 40503u + blockIdx.x * 97u;
  x ^= x >> 13;
  const unsigned ns = (x % 4u == 0) ? (x >> 20) % 8192u : 0u;
  if (ns) asm volatile("nanosleep.u32 %0;" ::"r"(ns));
#endif
}
__device__ __forceinline__ void fence_release() {
  jitter();
  asm volatile("fence.acq_rel" RESCCL_SC ";" ::: "memory");
}
// RESCCL_SPLIT_FENCE=1 (default): one-sided fences where one side suffices.  At .gpu / .sys
// scope the acquire half of a fence compiles to an L1 invalidate (CCTL.IVALL).
//   fence_rel: orders this thread's earlier reads and writes before its later stores (the
//     flag / credit / counter posts after a micro-batch's data moved): MEMBAR + ERRBAR, no
//     invalidate.
//   ready_ge: after a relaxed load observed a released value, fence.acquire orders it before
//     this thread's later reads (the PTX acquire pattern: strong read, then fence.acquire)
//     in place of a second, acquiring load of the same word.
// Both are the minimal orderings the protocol needs; on the device clock they measure the
// same as the two-sided forms (the per-primitive cost is not a cache effect).
#ifndef RESCCL_SPLIT_FENCE
#define RESCCL_SPLIT_FENCE 1
#endif
__device__ __forceinline__ void fence_rel() {
#if RESCCL_SPLIT_FENCE
  jitter();
  asm volatile("fence.release" RESCCL_SC ";" ::: "memory");
#else
  fence_release();
#endif
}
__device__ __forceinline__ u64 ld_acquire(const u64* p) {
  const u64 v = ld_acquire_raw(p);
#if RESCCL_JITTER
  jitter();
#endif
  return v;
}
// Polling: relaxed loads (an ld.acquire at .gpu/.sys scope compiles to a strong load plus
// an L1 invalidate, CCTL.IVALL, on every spin), then one acquire load once the value is
// reached: coherence makes it return a value >= the one observed, and it synchronises
// with the producer's release (fence + store) of that value.
__device__ __forceinline__ u64 ld_relaxed(const u64* p) {
  u64 v;
  asm volatile("ld.relaxed" RESCCL_SC ".global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
#ifndef RESCCL_POLL_ACQ
#define RESCCL_POLL_ACQ 0
#endif
// RESCCL_POLL_ACQ=1: every probe is the acquire load (one L2 round trip less per handoff
// once the value is there, an L1 invalidate per probe)
__device__ __forceinline__ bool ready_ge(const u64* p, u64 target) {
#if RESCCL_POLL_ACQ
  return ld_acquire(p) >= target;
#elif RESCCL_SPLIT_FENCE
  if (ld_relaxed(p) < target) return false;
  asm volatile("fence.acquire" RESCCL_SC ";" ::: "memory");
  jitter();
  return true;
#else
  if (ld_relaxed(p) < target) return false;
  (void)ld_acquire(p);
  return true;
#endif
}
__device__ __forceinline__ u64 globaltimer() {
  u64 t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#ifndef RESCCL_BACKOFF
#define RESCCL_BACKOFF 1
#endif
// polling back-off (RESCCL_BACKOFF=0: pure spin)
__device__ __forceinline__ void nanosleep_(u32 ns) {
#if RESCCL_BACKOFF
  asm volatile("nanosleep.u32 %0;" ::"r"(ns));
#endif
}

struct V4 {
  u32 x, y, z, w;
};
__device__ __forceinline__ V4 lds_v4(u32 a) {
  V4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_v4(u32 a, const V4& v) {
  asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ V4 ld_cg(const V4* p) {
  V4 v;
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ void st_v4(V4* p, const V4& v) {
  asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ u32 ld_cg_b32(const void* p) {
  u32 v;
  asm volatile("ld.global.cg.b32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ u16 ld_cg_b16(const void* p) {
  u16 v;
  asm volatile("ld.global.cg.b16 %0, [%1];" : "=h"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ void st_b32(void* p, u32 v) { asm volatile("st.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory"); }
__device__ __forceinline__ void st_b16(void* p, u16 v) { asm volatile("st.global.b16 [%0], %1;" ::"l"(p), "h"(v) : "memory"); }

// ----------------------------------------------------------------------------- TMA bulk copies
// cp.async.bulk global -> shared (mbarrier complete_tx) and shared -> global (bulk
// groups).  Used for the pure data-movement primitives (send, recv, rcs, rs, copy):
// one elected thread per lane keeps up to RESCCL_TMA_STAGES tiles in flight, so the
// bytes in flight per SM no longer depend on the thread count.
#ifndef RESCCL_TMA_TILE
#define RESCCL_TMA_TILE 16384
#endif
#ifndef RESCCL_TMA_STAGES
#define RESCCL_TMA_STAGES 4
#endif
__device__ __forceinline__ u32 smem_u32(const void* p) {
  return (u32)__cvta_generic_to_shared(p);
}
// shared-memory state through 32-bit shared addresses (generic pointers would compile to
// generic strong loads / GPU-scope atomics)
__device__ __forceinline__ u32 lds_u32(u32 a) {
  u32 v;
  asm volatile("ld.volatile.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_u32(u32 a, u32 v) {
  asm volatile("st.volatile.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ u64 lds_u64(u32 a) {
  u64 v;
  asm volatile("ld.volatile.shared.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_u64(u32 a, u64 v) {
  asm volatile("st.volatile.shared.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}
__device__ __forceinline__ u32 lds_u8(u32 a) {
  u32 v;
  asm volatile("ld.volatile.shared.u8 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_u8(u32 a, u32 v) {
  asm volatile("st.volatile.shared.u8 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ u32 atoms_and(u32 a, u32 v) {
  u32 old;
  asm volatile("atom.shared.and.b32 %0, [%1], %2;" : "=r"(old) : "r"(a), "r"(v) : "memory");
  return old;
}
__device__ __forceinline__ void atoms_or(u32 a, u32 v) {
  asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void fence_cta() { asm volatile("fence.acq_rel.cta;" ::: "memory"); }
__device__ __forceinline__ void mbar_init(u32 bar, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(u32 bar, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(u32 bar, u32 parity) {
  asm volatile(
      "{\n.reg .pred p;\nWAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n}\n" ::"r"(bar), "r"(parity) : "memory");
}
__device__ __forceinline__ bool mbar_test(u32 bar, u32 parity) {
  u32 ok;
  asm volatile(
      "{\n.reg .pred p;\n"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      "selp.u32 %0, 1, 0, p;\n}\n" : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
  return ok != 0;
}
// one suspending wait: the warp sleeps in hardware until the phase completes or a
// system-dependent time limit passes (no issue slots or smem bandwidth spent polling)
__device__ __forceinline__ bool mbar_try(u32 bar, u32 parity) {
  u32 ok;
  asm volatile(
      "{\n.reg .pred p;\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      "selp.u32 %0, 1, 0, p;\n}\n" : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_arrive(u32 bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
// wait until at most n bulk groups are pending (n must be an immediate)
__device__ __forceinline__ void tma_wait_n(u32 n) {
  switch (n < 15 ? n : 15) {
    case 1: asm volatile("cp.async.bulk.wait_group 1;" ::: "memory"); break;
    case 2: asm volatile("cp.async.bulk.wait_group 2;" ::: "memory"); break;
    case 3: asm volatile("cp.async.bulk.wait_group 3;" ::: "memory"); break;
    case 4: asm volatile("cp.async.bulk.wait_group 4;" ::: "memory"); break;
    case 5: asm volatile("cp.async.bulk.wait_group 5;" ::: "memory"); break;
    case 6: asm volatile("cp.async.bulk.wait_group 6;" ::: "memory"); break;
    case 7: asm volatile("cp.async.bulk.wait_group 7;" ::: "memory"); break;
    case 8: asm volatile("cp.async.bulk.wait_group 8;" ::: "memory"); break;
    case 9: asm volatile("cp.async.bulk.wait_group 9;" ::: "memory"); break;
    case 10: asm volatile("cp.async.bulk.wait_group 10;" ::: "memory"); break;
    case 11: asm volatile("cp.async.bulk.wait_group 11;" ::: "memory"); break;
    case 12: asm volatile("cp.async.bulk.wait_group 12;" ::: "memory"); break;
    case 13: asm volatile("cp.async.bulk.wait_group 13;" ::: "memory"); break;
    case 14: asm volatile("cp.async.bulk.wait_group 14;" ::: "memory"); break;
    case 15: asm volatile("cp.async.bulk.wait_group 15;" ::: "memory"); break;
    default: asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); break;
  }
}
__device__ __forceinline__ void tma_wait_read_n(u32 n) {
  switch (n < 15 ? n : 15) {
    case 1: asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory"); break;
    case 2: asm volatile("cp.async.bulk.wait_group.read 2;" ::: "memory"); break;
    case 3: asm volatile("cp.async.bulk.wait_group.read 3;" ::: "memory"); break;
    case 4: asm volatile("cp.async.bulk.wait_group.read 4;" ::: "memory"); break;
    case 5: asm volatile("cp.async.bulk.wait_group.read 5;" ::: "memory"); break;
    case 6: asm volatile("cp.async.bulk.wait_group.read 6;" ::: "memory"); break;
    case 7: asm volatile("cp.async.bulk.wait_group.read 7;" ::: "memory"); break;
    case 8: asm volatile("cp.async.bulk.wait_group.read 8;" ::: "memory"); break;
    case 9: asm volatile("cp.async.bulk.wait_group.read 9;" ::: "memory"); break;
    case 10: asm volatile("cp.async.bulk.wait_group.read 10;" ::: "memory"); break;
    case 11: asm volatile("cp.async.bulk.wait_group.read 11;" ::: "memory"); break;
    case 12: asm volatile("cp.async.bulk.wait_group.read 12;" ::: "memory"); break;
    case 13: asm volatile("cp.async.bulk.wait_group.read 13;" ::: "memory"); break;
    case 14: asm volatile("cp.async.bulk.wait_group.read 14;" ::: "memory"); break;
    case 15: asm volatile("cp.async.bulk.wait_group.read 15;" ::: "memory"); break;
    default: asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); break;
  }
}
// L2 eviction priorities (createpolicy): FIFO slots are written with evict_last so they
// stay L2-resident between producer and consumer; streamed user data and consumed FIFO
// payloads use evict_first (RESCCL_L2HINT, default on).
#ifndef RESCCL_L2HINT
#define RESCCL_L2HINT 1
#endif
__device__ __forceinline__ u64 policy_evict_first() {
  u64 p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ u64 policy_evict_last() {
  u64 p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void tma_load(u32 dst_smem, const void* src, u32 bytes, u32 bar, u64 pol) {
#if RESCCL_L2HINT
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
      ::"r"(dst_smem), "l"(src), "r"(bytes), "r"(bar), "l"(pol) : "memory");
#else
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(dst_smem), "l"(src), "r"(bytes), "r"(bar) : "memory");
#endif
}
__device__ __forceinline__ void tma_store(void* dst, u32 src_smem, u32 bytes, u64 pol) {
#if RESCCL_L2HINT
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;"
               ::"l"(dst), "r"(src_smem), "r"(bytes), "l"(pol) : "memory");
#else
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src_smem), "r"(bytes)
               : "memory");
#endif
}
#ifndef RESCCL_PREFETCH
#define RESCCL_PREFETCH 0
#endif
// Bulk prefetch of local HBM data into L2 (no shared memory involved).  L2 is the
// device's point of coherence, so prefetching a slice before its producer finished
// is safe: later writes update the L2 lines.
__device__ __forceinline__ void l2_prefetch(const void* p, u32 bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void tma_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void tma_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }

// ----------------------------------------------------------------------------- element types
// Storage types: int32 / f32 as 32-bit words, f16 / bf16 as 16-bit words.
struct TI32 { enum { kSize = 4, kKind = 0 }; };
struct TF32 { enum { kSize = 4, kKind = 1 }; };
struct TF16 { enum { kSize = 2, kKind = 2 }; };
struct TBF16 { enum { kSize = 2, kKind = 3 }; };

__device__ __forceinline__ float bf_lo(u32 w) { return __uint_as_float(w << 16); }
__device__ __forceinline__ float bf_hi(u32 w) { return __uint_as_float(w & 0xFFFF0000u); }
__device__ __forceinline__ u32 pack_bf16x2(float lo, float hi) {
  u32 r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}
__device__ __forceinline__ float h_lo(u32 w) {
  float f;
  asm("{.reg .b16 l, h; mov.b32 {l, h}, %1; cvt.f32.f16 %0, l;}" : "=f"(f) : "r"(w));
  return f;
}
__device__ __forceinline__ float h_hi(u32 w) {
  float f;
  asm("{.reg .b16 l, h; mov.b32 {l, h}, %1; cvt.f32.f16 %0, h;}" : "=f"(f) : "r"(w));
  return f;
}
__device__ __forceinline__ u32 pack_f16x2(float lo, float hi) {
  u32 r;
  asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}
__device__ __forceinline__ float bf16_to_f(u16 h) { return __uint_as_float(((u32)h) << 16); }
__device__ __forceinline__ u16 f_to_bf16(float f) {
  u16 r;
  asm("cvt.rn.bf16.f32 %0, %1;" : "=h"(r) : "f"(f));
  return r;
}
__device__ __forceinline__ float f16_to_f(u16 h) {
  float f;
  asm("cvt.f32.f16 %0, %1;" : "=f"(f) : "h"(h));
  return f;
}
__device__ __forceinline__ u16 f_to_f16(float f) {
  u16 r;
  asm("cvt.rn.f16.f32 %0, %1;" : "=h"(r) : "f"(f));
  return r;
}

template <int OP>
__device__ __forceinline__ float fop(float a, float b) {
  if (OP == OpSum) return __fadd_rn(a, b);
  if (OP == OpMax) return fmaxf(a, b);
  return fminf(a, b);
}
template <int OP>
__device__ __forceinline__ u32 iop(u32 a, u32 b) {
  if (OP == OpSum) return a + b;  // two's-complement wraparound
  if (OP == OpMax) return (u32)max((int)a, (int)b);
  return (u32)min((int)a, (int)b);
}

// combine one 32-bit word: local (+) incoming
template <class T, int OP>
__device__ __forceinline__ u32 combine_w(u32 a, u32 b);
template <> __device__ __forceinline__ u32 combine_w<TI32, OpSum>(u32 a, u32 b) { return iop<OpSum>(a, b); }
template <> __device__ __forceinline__ u32 combine_w<TI32, OpMax>(u32 a, u32 b) { return iop<OpMax>(a, b); }
template <> __device__ __forceinline__ u32 combine_w<TI32, OpMin>(u32 a, u32 b) { return iop<OpMin>(a, b); }
#define RDEV_F32(OPV) \
  template <> __device__ __forceinline__ u32 combine_w<TF32, OPV>(u32 a, u32 b) { \
    return __float_as_uint(fop<OPV>(__uint_as_float(a), __uint_as_float(b))); }
RDEV_F32(OpSum) RDEV_F32(OpMax) RDEV_F32(OpMin)
#undef RDEV_F32
#define RDEV_BF(OPV) \
  template <> __device__ __forceinline__ u32 combine_w<TBF16, OPV>(u32 a, u32 b) { \
    return pack_bf16x2(fop<OPV>(bf_lo(a), bf_lo(b)), fop<OPV>(bf_hi(a), bf_hi(b))); }
RDEV_BF(OpMax) RDEV_BF(OpMin)
#undef RDEV_BF
#define RDEV_H(OPV) \
  template <> __device__ __forceinline__ u32 combine_w<TF16, OPV>(u32 a, u32 b) { \
    return pack_f16x2(fop<OPV>(h_lo(a), h_lo(b)), fop<OPV>(h_hi(a), h_hi(b))); }
RDEV_H(OpMax) RDEV_H(OpMin)
#undef RDEV_H
// 16-bit sums: one packed add, correctly rounded (RN, subnormals kept) -- the value R8
// fixes (binary32 add then RNE equals the correctly rounded 16-bit add)
template <> __device__ __forceinline__ u32 combine_w<TBF16, OpSum>(u32 a, u32 b) {
  u32 r;
  asm("add.rn.bf16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}
template <> __device__ __forceinline__ u32 combine_w<TF16, OpSum>(u32 a, u32 b) {
  u32 r;
  asm("add.rn.f16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}

template <class T, int OP>
__device__ __forceinline__ V4 combine_v(const V4& a, const V4& b) {
  V4 r;
  r.x = combine_w<T, OP>(a.x, b.x);
  r.y = combine_w<T, OP>(a.y, b.y);
  r.z = combine_w<T, OP>(a.z, b.z);
  r.w = combine_w<T, OP>(a.w, b.w);
  return r;
}

// scalar (one element) path for misaligned slices and vector tails
template <class T, int OP>
__device__ __forceinline__ void elem_move(int F, const char* A, const char* B, char* D1, char* D2, i64 i) {
  if (T::kSize == 4) {
    u32 a = 0, b = 0, v;
    if (A) a = ld_cg_b32(A + 4 * i);
    if (B) b = ld_cg_b32(B + 4 * i);
    v = (F & kReduce) ? combine_w<T, OP>(a, b) : ((F & kRecv) ? b : a);
    if (D1) st_b32(D1 + 4 * i, v);
    if (D2) st_b32(D2 + 4 * i, v);
  } else {
    u16 a = 0, b = 0, v;
    if (A) a = ld_cg_b16(A + 2 * i);
    if (B) b = ld_cg_b16(B + 2 * i);
    if (F & kReduce) {
      if (T::kKind == 3)
        v = f_to_bf16(fop<OP>(bf16_to_f(a), bf16_to_f(b)));
      else
        v = f_to_f16(fop<OP>(f16_to_f(a), f16_to_f(b)));
    } else {
      v = (F & kRecv) ? b : a;
    }
    if (D1) st_b16(D1 + 2 * i, v);
    if (D2) st_b16(D2 + 2 * i, v);
  }
}

// Move n elements: A = local source, B = incoming FIFO slot, D1 = local store target,
// D2 = outgoing FIFO slot.  Null pointers are unused operands (fixed per primitive).
template <class T, int OP, int F, int U>
__device__ __forceinline__ void move(i64 n, const char* A, const char* B, char* D1, char* D2, int tid, int nt) {
  if (n <= 0) return;
  const unsigned long long al = (unsigned long long)A | (unsigned long long)B | (unsigned long long)D1 |
                                (unsigned long long)D2;
  const i64 bytes = n * T::kSize;
  i64 nv = 0;
  if ((al & 15) == 0) {
    nv = bytes >> 4;
    const V4* a4 = (const V4*)A;
    const V4* b4 = (const V4*)B;
    V4* d1 = (V4*)D1;
    V4* d2 = (V4*)D2;
    i64 i = tid;
    // main body: U independent 16-byte vectors in flight per operand per thread
    for (; i + (i64)(U - 1) * nt < nv; i += (i64)U * nt) {
      V4 va[U], vb[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (A) va[u] = ld_cg(a4 + i + (i64)u * nt);
        if (B) vb[u] = ld_cg(b4 + i + (i64)u * nt);
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        V4 v = (F & kReduce) ? combine_v<T, OP>(va[u], vb[u]) : ((F & kRecv) ? vb[u] : va[u]);
        if (D1) st_v4(d1 + i + (i64)u * nt, v);
        if (D2) st_v4(d2 + i + (i64)u * nt, v);
      }
    }
    for (; i < nv; i += nt) {
      V4 va, vb;
      if (A) va = ld_cg(a4 + i);
      if (B) vb = ld_cg(b4 + i);
      V4 v = (F & kReduce) ? combine_v<T, OP>(va, vb) : ((F & kRecv) ? vb : va);
      if (D1) st_v4(d1 + i, v);
      if (D2) st_v4(d2 + i, v);
    }
  }
  const i64 e0 = (nv << 4) / T::kSize;
  for (i64 e = e0 + tid; e < n; e += nt) elem_move<T, OP>(F, A, B, D1, D2, e);
}

// ----------------------------------------------------------------------------- lane
// RESCCL_LOOKAHEAD (DESIGN R30): a lane leader posts the "writable" credits of its
// upcoming push receives (direct transport) as soon as their dependencies hold, from any
// idle poll, instead of when the lane reaches them.
#if !defined(RESCCL_K)  // no plan layout (the NVLS-only self-test): no primitives either
#undef RESCCL_LOOKAHEAD
#define RESCCL_LOOKAHEAD 0
#endif
#ifndef RESCCL_LOOKAHEAD
#define RESCCL_LOOKAHEAD 1
#endif
struct Lane;
struct PrimDesc;
template <int U = 0>
__device__ __noinline__ void lookahead(Lane& L);

struct Lane {
  const KArgs* a;
  char* self;       // this rank's plan region
  int rank, inst, bar, nthreads, tid;
  volatile int* abort_flag;  // shared memory, per lane
  // shared-memory addresses (32-bit):
  u32 stage;                 // the CTA's stage pool: RESCCL_POOL x (A tile, B tile), shared by both lanes
  u32 full;                  // "tile loaded" mbarriers (one per pool stage)
  u32 comp;                  // "tile combined" mbarriers (one per pool stage)
  u32 pool;                  // u32 mask: bit s set = pool stage s free
  u32 qprog;                 // u32: tiles this lane's leader announced to its combine warps
  u32 qdesc;                 // u64: the current epoch (first tile | stage mask << 32 | parities << 48)
  u32 want;                  // u32[2]: lane waits for pool stages (send lane, recv lane)
  u32 tseq;                  // tiles streamed so far by this lane
  u32 ring0;                 // RESCCL_RING: first stage of this lane's private ring
  u32 cpar;                  // RESCCL_RING (leader): comp-barrier phase parity per ring slot
  u64 wait_ns;               // RESCCL_TRACE: leader time spent waiting (idle ratio, Table 3)
  int pidx;                  // index of the running primitive in the rank's descriptor table
  u64* ph;                   // RESCCL_PHASE: this lane's record area (null: off)
  u32 nph;                   // RESCCL_PHASE: records written
  u64 t_run;                 // RESCCL_PHASE: entry of the running primitive (before its setup)
  u64 t_call;                // RESCCL_PHASE: the generated code reached the primitive's call
  u64 t_pro;                 // RESCCL_PHASE: entry of the engine function (after run's setup)
  u64 t_end;                 // RESCCL_PHASE: the previous primitive's engine function returned
  // writable lookahead (leader): the lane's push receives in lane order (descriptor index,
  // gate = 1 + lane index of the last earlier same-lane primitive a dropped implied
  // dependency pointed at), the cursor (push receive wa_c, micro-batch wa_m) of the next
  // credit to post, the lane index of the running primitive and its push-receive index
  u32 cta_idle;              // RESCCL_TRACE (smem): u32 lanes idle, u32 pad, u64 both-idle ns, u64 start[2]
  const PrimDesc* descs;
  const int* wa;
  const int* wg;
  int wa_n, wa_c, wa_m, lpos, wai;

  __device__ __forceinline__ void sync() const {
    asm volatile("barrier.sync %0, %1;" ::"r"(bar), "r"(nthreads) : "memory");  // (divergence-tolerant)
  }
  // leader only: spin until *p >= target; false on timeout (error word set)
  __device__ bool wait_ge(const u64* p, u64 target) {
    if (ready_ge(p, target)) return true;
    u64 t0 = globaltimer();
#if RESCCL_TRACE
    cta_idle_enter_(t0);
#endif
    u32 spins = 0;
    while (!ready_ge(p, target)) {
#if RESCCL_LOOKAHEAD
      if (wa_c < wa_n && (spins & 7) == 7) lookahead<0>(*this);  // rate-limited: the wait's own poll first
#endif
      if (++spins > 64) nanosleep_(32);
      if ((spins & 1023) == 0 && globaltimer() - t0 > a->timeout_ns) {
        atomicCAS(a->err, 0, kErrTimeout);
        return false;
      }
    }
#if RESCCL_TRACE
    const u64 t1 = globaltimer();
    wait_ns += t1 - t0;
    cta_idle_exit_(t1);
#endif
    return true;
  }
  __device__ void cta_idle_enter_(u64 now);
  __device__ void cta_idle_exit_(u64 now);
};

__device__ __forceinline__ u64* at(char* base, i64 off) { return (u64*)(base + off); }

// RESCCL_TRACE: a lane leader's busy-waiting intervals (waiting for a peer's flag or
// credit or for a local dependency, with no data of its own in flight).  Per lane they sum
// to wait_ns (the paper's per-TB idle ratio, with a lane as the paper's TB);
// per CTA the intervals in which BOTH lanes busy-wait (or have finished) are summed in
// shared memory: the SM itself is then occupied without moving data.
__device__ __forceinline__ void cta_idle_enter(const Lane& L, u64 now) {
#if RESCCL_TRACE
  sts_u64(L.cta_idle + 16 + 8 * (L.bar - 1), now);  // this lane's start, before the count
  fence_cta();
  asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(L.cta_idle) : "memory");
#endif
}
__device__ __forceinline__ void cta_idle_exit(const Lane& L, u64 now) {
#if RESCCL_TRACE
  u32 old;
  asm volatile("atom.shared.add.u32 %0, [%1], -1;" : "=r"(old) : "r"(L.cta_idle) : "memory");
  if (old == 2) {  // both lanes were idle: from the later of the two starts until now
    const u64 a0 = lds_u64(L.cta_idle + 16), a1 = lds_u64(L.cta_idle + 24);
    const u64 st = a0 > a1 ? a0 : a1;
    if (now > st) {
      const u32 addr = L.cta_idle + 8;
      const u64 d = now - st;
      asm volatile("red.shared.add.u64 [%0], %1;" ::"r"(addr), "l"(d) : "memory");
    }
  }
#endif
}
__device__ __forceinline__ void Lane::cta_idle_enter_(u64 now) { cta_idle_enter(*this, now); }
__device__ __forceinline__ void Lane::cta_idle_exit_(u64 now) { cta_idle_exit(*this, now); }
__device__ __forceinline__ void idle_on(Lane& L, u64& t_idle) {
#if RESCCL_TRACE
  if (t_idle == 0) {
    t_idle = globaltimer();
    cta_idle_enter(L, t_idle);
  }
#endif
}
__device__ __forceinline__ void idle_off(Lane& L, u64& t_idle) {
#if RESCCL_TRACE
  if (t_idle) {
    const u64 now = globaltimer();
    L.wait_ns += now - t_idle;
    cta_idle_exit(L, now);
  }
#endif
  t_idle = 0;
}

// RESCCL_PHASE record (leader only): kind 0 = blocking register path, 1 = flag-only
// primitive, 2 = TMA lane engine; t[0..4] as documented at each call site.
enum : int { PhSync = 0, PhFlags = 1, PhPipe = 2 };
__device__ __forceinline__ void ph_rec(Lane& L, int kind, int j, u64 t0, u64 t1, u64 t2, u64 t3, u64 t4) {
#if RESCCL_PHASE
  if (!L.ph || L.nph + 1 >= RESCCL_PH_MAX) return;
  u64* r = L.ph + 8 * (size_t)(++L.nph);
  r[0] = ((u64)(u32)L.pidx << 32) | ((u64)(u32)j << 8) | (u64)kind;
  r[1] = t0;
  r[2] = t1;
  r[3] = t2;
  r[4] = t3;
  r[5] = t4;
  r[6] = L.t_call;
  // ns deltas, 16 bits each (saturating): run entry - call, engine entry - run entry,
  // call - previous primitive's return
  auto d16 = [](u64 a, u64 b) -> u64 { return (a && b && a >= b) ? (a - b > 65535 ? 65535 : a - b) : 65535; };
  r[7] = d16(L.t_run, L.t_call) | (d16(L.t_pro, L.t_run) << 16) | (d16(L.t_call, L.t_end) << 32);
#else
  (void)L; (void)kind; (void)j; (void)t0; (void)t1; (void)t2; (void)t3; (void)t4;
#endif
}
__device__ __forceinline__ u64 ph_now() {
#if RESCCL_PHASE
  return globaltimer();
#else
  return 0;
#endif
}
// generated call sites stamp the moment the lane's code reaches a primitive's call
#if RESCCL_PHASE
#define RESCCL_PH_CALL(L) ((L).t_call = rdev::globaltimer())
#else
#define RESCCL_PH_CALL(L) ((void)0)
#endif

template <int COLL>
__device__ __forceinline__ i64 chunk_len(const KArgs& a, int c) {
  if (COLL == CollAllReduce) {
    i64 l = a.count - (i64)c * a.C;
    return l < 0 ? 0 : (l > a.C ? a.C : l);
  }
  return a.count;
}
template <int COLL>
__device__ __forceinline__ i64 chunk_off(int buf, int c, i64 C) {
  if (COLL == CollAllReduce) return (i64)c * C;
  if (COLL == CollAllGather) return buf == BufSend ? 0 : (i64)c * C;
  return buf == BufRecv ? 0 : (i64)c * C;  // reduce-scatter
}
__device__ __forceinline__ char* buf_ptr(const KArgs& a, int rank, int buf) {
  return buf == BufSend ? (char*)a.sendbuf[rank] : (buf == BufRecv ? a.recvbuf[rank] : a.scratch[rank]);
}

// One primitive of the schedule: constants emitted by the kernel generator as a
// literal.  Offsets are bytes inside the plan region of the named rank's arena, for
// instance 0 (instance i adds i * K * SLOT, i * FLAGSTRIDE or i * 128).
#ifndef RESCCL_MAXDEPS
#define RESCCL_MAXDEPS 6
#endif
struct PrimDesc {
  int chunk, src_buf, dst_buf, in_peer, out_peer, ndeps;
  i64 in_data, in_flag, in_cred, in_pos, in_n;
  i64 out_data, out_flag, out_cred, out_pos, out_n;
  i64 ctr;
  int rem_rank, rem_buf;       // direct mode: the peer location a pull reads
  int out_rank, out_buf;       // direct mode: the peer location a push writes
  // dependency k is satisfied for micro-batch j when the u64 at deps[k] in this rank's
  // region reaches dep_n[k] * mb_base + dep_pos[k] * n_mb + j + 1: a completion counter
  // (n = 1, pos = 0) or, for a direct pull-send, the receiver's read credit of its link.
  i64 deps[RESCCL_MAXDEPS];
  i64 dep_n[RESCCL_MAXDEPS];
  i64 dep_pos[RESCCL_MAXDEPS];
  // bit k: dependency k is a flag ring slot instead of a counter -- the "written" flag of
  // a flags-only push receive (drecv / drecv_p) on this rank, awaited directly instead of
  // the counter that receive posts once it saw the flag (relay bypass, DESIGN R29): deps[k]
  // is then the ring's offset, the slot is (target - 1) % K, the stride per instance
  // RESCCL_FLAGSTRIDE
  int dep_ring;
};

// Layout constants shared by every primitive of a plan (emitted by the generator):
//   RESCCL_K, RESCCL_I, RESCCL_SLOT, RESCCL_FLAGSTRIDE, RESCCL_COLL
struct PrimPtrs {
  const char* A;     // local operand base (chunk start)
  char* D1;          // local store target base (chunk start)
  char* in_data;     // incoming FIFO slots (this instance)
  u64* in_flag;
  u64* in_cred;      // credit counter in the sender's arena
  char* out_data;    // outgoing FIFO slots in the receiver's arena
  u64* out_flag;
  u64* out_cred;     // credit counter the receiver writes back (own arena)
  u64* ctr;
  const char* R;     // direct mode: pulled peer location base (chunk start)
  char* Q;           // direct mode: pushed peer location base (chunk start)
  i64 len;           // chunk length (elements)
};

// primitive anatomy (compile-time, from the flags)
template <int F> struct Kind {
  static constexpr bool push_recv = (F & kDirect) && (F & kRecv) && !(F & kPull);  // payload pushed to us
  static constexpr bool has_b = (F & kRecv) && !push_recv;             // incoming operand: FIFO slot / pulled
  static constexpr bool send_data = (F & kSend) && !((F & kDirect) && (F & kSendPull));  // we write the payload
  static constexpr int mf = (F & kReduce) | (has_b ? kRecv : 0);      // value = A (+) B, B, or A
};

// RESCCL_BULKRED: an in-place reduce primitive (local location == store target, nothing
// forwarded) streams only the incoming tile into shared memory and adds it into the local
// buffer with one bulk reduction (cp.reduce.async.bulk ... .add, done in L2): no local
// tile in shared memory and no combine warps.  One correctly rounded add of `local` and
// `incoming` per element -- the same value as R8's combine (bf16/fp16 .noftz, RN).  f32
// max/min have no bulk form and keep the combine path.
#ifndef RESCCL_BULKRED
#define RESCCL_BULKRED 0
#endif
template <class T, int OP>
struct BulkRed { static constexpr bool ok = !(T::kKind == 1 && OP != OpSum); };
template <class T, int OP>
__device__ __forceinline__ void tma_reduce(void* dst, u32 src_smem, u32 bytes, u64 pol);
#define RESCCL_BRED(TT, O, SUF)                                                                          \
  template <>                                                                                            \
  __device__ __forceinline__ void tma_reduce<TT, O>(void* dst, u32 src, u32 bytes, u64 pol) {            \
    asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.L2::cache_hint." SUF " [%0], [%1], %2, %3;" \
                 ::"l"(dst), "r"(src), "r"(bytes), "l"(pol) : "memory");                                 \
  }
RESCCL_BRED(TBF16, OpSum, "add.noftz.bf16")
RESCCL_BRED(TBF16, OpMax, "max.bf16")
RESCCL_BRED(TBF16, OpMin, "min.bf16")
RESCCL_BRED(TF16, OpSum, "add.noftz.f16")
RESCCL_BRED(TF16, OpMax, "max.f16")
RESCCL_BRED(TF16, OpMin, "min.f16")
RESCCL_BRED(TF32, OpSum, "add.f32")
RESCCL_BRED(TI32, OpSum, "add.u32")
RESCCL_BRED(TI32, OpMax, "max.s32")
RESCCL_BRED(TI32, OpMin, "min.s32")
#undef RESCCL_BRED
template <> __device__ __forceinline__ void tma_reduce<TF32, OpMax>(void*, u32, u32, u64) { __trap(); }
template <> __device__ __forceinline__ void tma_reduce<TF32, OpMin>(void*, u32, u32, u64) { __trap(); }
// does this reduce primitive take the bulk-reduction path? (leader and combine warps agree)
template <class T, int OP, int F>
__device__ __forceinline__ bool bulk_reduce_prim(const char* A, const char* D1) {
  return RESCCL_BULKRED && (F & kReduce) && (F & kStore) && !Kind<F>::send_data && BulkRed<T, OP>::ok &&
         A != nullptr && A == D1;
}

__device__ __forceinline__ u64 dep_target(const KArgs& a, const PrimDesc& d, int k, int j) {
  return (u64)d.dep_n[k] * a.mb_base + (u64)d.dep_pos[k] * a.n_mb + j + 1;
}
// the u64 dependency k of micro-batch j waits on (see PrimDesc::dep_ring); templates so
// that the plan's layout macros (RESCCL_K, RESCCL_FLAGSTRIDE) are needed only when used
template <int U = 0>
__device__ __forceinline__ const u64* dep_ptr(char* self, int inst, const PrimDesc& d, int k, u64 target) {
  if (d.dep_ring & (1 << k))
    return at(self, d.deps[k] + (i64)inst * RESCCL_FLAGSTRIDE + (i64)((target - 1) % RESCCL_K) * 8);
  return at(self, d.deps[k] + (i64)inst * 128);
}
template <int U = 0>
__device__ __forceinline__ bool dep_ready(const Lane& L, const PrimDesc& d, int k, int j) {
  const u64 t = dep_target(*L.a, d, k, j);
  return ready_ge(dep_ptr<U>(L.self, L.inst, d, k, t), t);
}
// relaxed observation only: for waits followed by fence_release() (fence.acq_rel), which
// acquires what was observed -- no confirming acquire load (one L2 round trip less)
template <int U = 0>
__device__ __forceinline__ bool dep_seen(const Lane& L, const PrimDesc& d, int k, int j) {
  const u64 t = dep_target(*L.a, d, k, j);
  return ld_relaxed(dep_ptr<U>(L.self, L.inst, d, k, t)) >= t;
}

// Post at most one "writable" credit: the next one of the lane's push receives, if the
// lane has passed every earlier same-lane primitive it depends on (gate) and its explicit
// dependencies hold for that micro-batch -- the same conditions the primitive itself
// checks when the lane reaches it, so the credit only comes earlier (monotone flags: no
// new wait edge, DESIGN R30).  Leader thread only.
template <int U>
__device__ __noinline__ void lookahead(Lane& L) {
  const KArgs& a = *L.a;
  while (L.wa_c < L.wa_n) {
    if (L.wa_m >= a.n_mb) {
      ++L.wa_c;
      L.wa_m = 0;
      continue;
    }
    if (L.lpos < L.wg[L.wa_c]) return;
    const PrimDesc& d = L.descs[L.wa[L.wa_c]];
    const u64 in_seq = (u64)d.in_n * a.mb_base + (u64)d.in_pos * a.n_mb + L.wa_m;
    u64* const cred = at(a.arena[d.in_peer], d.in_cred + (i64)L.inst * 128);
    // every probe is a relaxed load issued before any is tested (one L2 round trip in
    // all); the fence.acq_rel before the post acquires what they observed.  The link's
    // credit is one monotone counter for every position on the link (push "writable" and
    // pull "read" alike): "credit >= pos + 1" must imply every earlier position was
    // credited, so this one waits until the previous sequence was posted (by this lane or
    // by another lane receiving on the same link)
    u64 v[RESCCL_MAXDEPS], tg[RESCCL_MAXDEPS];
#pragma unroll
    for (int k = 0; k < RESCCL_MAXDEPS; ++k)
      if (k < d.ndeps) {
        tg[k] = dep_target(a, d, k, L.wa_m);
        v[k] = ld_relaxed(dep_ptr<U>(L.self, L.inst, d, k, tg[k]));
      }
    const u64 c = ld_relaxed(cred);
#pragma unroll
    for (int k = 0; k < RESCCL_MAXDEPS; ++k)
      if (k < d.ndeps && v[k] < tg[k]) return;
    if (c < in_seq) return;
    fence_release();
    st_relaxed(cred, in_seq + 1);
    ++L.wa_m;
    return;
  }
}
// micro-batches of the running push receive whose "writable" is posted
__device__ __forceinline__ int writable_posted(const Lane& L, int nmb) {
  return L.wa_c > L.wai ? nmb : (L.wa_c == L.wai ? L.wa_m : 0);
}

__device__ __forceinline__ void slice_of(const KArgs& a, i64 len, int j, int inst, i64& lo, i64& hi) {
  lo = (i64)j * a.M + (i64)inst * a.Mi;
  hi = lo + a.Mi;
  if (hi > (i64)(j + 1) * a.M) hi = (i64)(j + 1) * a.M;
  if (hi > len) hi = len;
  if (lo > hi) lo = hi;
}

template <int F>
__device__ __forceinline__ void post_mb(const KArgs& a, const PrimDesc& d, const PrimPtrs& p, int j) {
  const u64 mb_base = a.mb_base;
  const u64 in_seq = (u64)d.in_n * mb_base + (u64)d.in_pos * a.n_mb + j;
  const u64 out_seq = (u64)d.out_n * mb_base + (u64)d.out_pos * a.n_mb + j;
  fence_rel();
  if (F & kSend) st_relaxed(p.out_flag + (out_seq % RESCCL_K), out_seq + 1);   // payload / written / readable
  if (Kind<F>::has_b) st_relaxed(p.in_cred, in_seq + 1);                        // consumed / read (push: posted earlier)
  if (d.ctr >= 0) st_relaxed(p.ctr, mb_base + j + 1);
}

template <int F>
__device__ __forceinline__ void post_writable(const KArgs& a, const PrimDesc& d, const PrimPtrs& p, int j) {
  const u64 in_seq = (u64)d.in_n * a.mb_base + (u64)d.in_pos * a.n_mb + j;
  fence_rel();
  st_relaxed(p.in_cred, in_seq + 1);
}

// Non-blocking readiness of micro-batch j: local dependencies, payload, credit.
template <int F>
__device__ __forceinline__ bool mb_ready(const Lane& L, const PrimDesc& d, const PrimPtrs& p, int j) {
  const KArgs& a = *L.a;
  const u64 mb_base = a.mb_base;
  if (!Kind<F>::push_recv)  // (a push receiver checked its dependencies when it posted "writable")
    for (int k = 0; k < d.ndeps; ++k)
      if (!dep_ready(L, d, k, j)) return false;
  if (F & kRecv) {
    const u64 in_seq = (u64)d.in_n * mb_base + (u64)d.in_pos * a.n_mb + j;
    if (!ready_ge(p.in_flag + (in_seq % RESCCL_K), in_seq + 1)) return false;
  }
  if (F & kSend) {
    const u64 out_seq = (u64)d.out_n * mb_base + (u64)d.out_pos * a.n_mb + j;
    if (F & kDirect) {
      if (!(F & kSendPull) && !ready_ge(p.out_cred, out_seq + 1)) return false;  // push: writable
    } else if (out_seq + 1 > (u64)RESCCL_K && !ready_ge(p.out_cred, out_seq + 1 - RESCCL_K)) {
      return false;
    }
  }
  return true;
}

// Blocking per-micro-batch path (all lane threads; 16-byte LD/ST): used for misaligned
// buffers and when the TMA pipeline is disabled.
template <class T, int OP, int F>
__device__ __noinline__ bool run_sync(Lane& L, const PrimDesc& d, const PrimPtrs& p) {
  const KArgs& a = *L.a;
  const u64 mb_base = a.mb_base;
  for (int j = 0; j < a.n_mb; ++j) {
    const u64 in_seq = (u64)d.in_n * mb_base + (u64)d.in_pos * a.n_mb + j;
    const u64 out_seq = (u64)d.out_n * mb_base + (u64)d.out_pos * a.n_mb + j;
    // phase record: t0 start, t1 local dependencies met, t2 flag / credit met, t3 data
    // moved (lane barrier passed), t4 posted (fence + flag stores issued)
    u64 ph0 = 0, ph1 = 0, ph2 = 0;
    if (L.tid == 0) {
      ph0 = ph_now();
      bool ok = true;
#if RESCCL_LOOKAHEAD
      if (Kind<F>::push_recv) {  // the lane's writable cursor posts it (R30)
        const u64 t0 = globaltimer();
        u32 spins = 0;
        while (writable_posted(L, a.n_mb) <= j) {
          lookahead(L);
          if (writable_posted(L, a.n_mb) > j) break;
          if (++spins > 64) nanosleep_(32);
          if ((spins & 1023) == 0 && globaltimer() - t0 > a.timeout_ns) {
            atomicCAS(a.err, 0, kErrTimeout);
            ok = false;
            break;
          }
        }
      } else
#endif
        for (int k = 0; k < d.ndeps && ok; ++k)
          ok = L.wait_ge(dep_ptr(L.self, L.inst, d, k, dep_target(a, d, k, j)), dep_target(a, d, k, j));
      ph1 = ph_now();
#if !RESCCL_LOOKAHEAD
      if (ok && Kind<F>::push_recv) post_writable<F>(a, d, p, j);
#endif
      if (ok && (F & kRecv)) ok = L.wait_ge(p.in_flag + (in_seq % RESCCL_K), in_seq + 1);
      if (ok && (F & kSend)) {
        if (F & kDirect) {
          if (!(F & kSendPull)) ok = L.wait_ge(p.out_cred, out_seq + 1);
        } else if (out_seq + 1 > (u64)RESCCL_K) {
          ok = L.wait_ge(p.out_cred, out_seq + 1 - RESCCL_K);
        }
      }
      if (!ok) *L.abort_flag = 1;
      ph2 = ph_now();
    }
    L.sync();
    if (*L.abort_flag) return false;
    i64 lo, hi;
    slice_of(a, p.len, j, L.inst, lo, hi);
    const char* Aj = p.A ? p.A + lo * T::kSize : nullptr;
    char* D1j = p.D1 ? p.D1 + lo * T::kSize : nullptr;
    const char* Bj = Kind<F>::has_b ? ((F & kDirect) ? p.R + lo * T::kSize
                                                     : p.in_data + (in_seq % RESCCL_K) * RESCCL_SLOT)
                                    : nullptr;
    char* D2j = Kind<F>::send_data ? ((F & kDirect) ? p.Q + lo * T::kSize : p.out_data + (out_seq % RESCCL_K) * RESCCL_SLOT)
                                   : nullptr;
    move<T, OP, Kind<F>::mf, 4>(hi - lo, Aj, Bj, D1j, D2j, L.tid, L.nthreads);
    L.sync();
    if (L.tid == 0) {
      const u64 ph3 = ph_now();
      post_mb<F>(a, d, p, j);
      ph_rec(L, PhSync, j, ph0, ph1, ph2, ph3, ph_now());
    }
  }
  return true;
}

// Stage management.  A CTA owns RESCCL_POOL = 2 x RESCCL_TMA_STAGES TMA stages (an A
// and a B tile each).  In most schedules only one lane moves data at a time (ring
// AllReduce: the receive lane during ReduceScatter, the send lane during AllGather), so
// by default the lanes share the stages as a pool, claimed in *epochs*: a leader that has
// confirmed-ready work and no stages takes every free stage (at most half while the other
// lane waits for stages) with one shared-memory atomic, streams its tiles round-robin
// through them, and returns them once everything it loaded is written out and no ready
// work is left (or early, when the other lane waits and it holds more than half).
// Per tile the leader touches shared memory only through the TMA, its mbarriers and one
// progress word: its generic shared-memory operations queue behind the TMA's bulk smem
// traffic (~300 cycles each under load), so per-tile claims capped the tile rate.
// Deadlock freedom: a leader holds stages only while it has unposted tiles or confirmed-
// ready loads, both of which complete without any remote condition, so a leader waiting
// on a remote condition holds no stage and a lane waiting for stages waits only for the
// other lane's local work: no new wait edge.
// RESCCL_RING=1: each lane streams through a private ring of RESCCL_TMA_STAGES stages
// instead (tile k -> stage ring0 + k % S, full parity (k / S) & 1).
#define RESCCL_POOL (2 * RESCCL_TMA_STAGES)
#ifndef RESCCL_POOL_CAP
#define RESCCL_POOL_CAP RESCCL_POOL  // stages one lane may hold
#endif
#ifndef RESCCL_RING
#define RESCCL_RING 0
#endif
// combine warps: 1 = one warp polls the leader's progress word, the rest wait on a named
// barrier (ids 3 / 4 = the lane's barrier + 2)
#ifndef RESCCL_CPOLL
#define RESCCL_CPOLL 0
#endif
// stores a lane lets drain before it blocks on the oldest to reuse its stage
#ifndef RESCCL_STORE_LAG
#define RESCCL_STORE_LAG 1
#endif
// RESCCL_EARLY_EXIT=1 (default): the leader leaves its event loop right after the last post
#ifndef RESCCL_EARLY_EXIT
#define RESCCL_EARLY_EXIT 1
#endif
// parity of a quiescent mbarrier's current (incomplete) phase: the preceding phase, of
// the other parity, tests complete
__device__ __forceinline__ u32 mbar_phase(u32 bar) { return mbar_test(bar, 0) ? 1u : 0u; }
// i-th (0-based) set bit of m
__device__ __forceinline__ u32 nth_bit(u32 m, u32 i) {
  for (; i; --i) m &= m - 1;
  return (u32)(__ffs(m) - 1);
}

__device__ __forceinline__ void slice_of_m(i64 M, i64 Mi, i64 len, int j, int inst, i64& lo, i64& hi) {
  lo = (i64)j * M + (i64)inst * Mi;
  hi = lo + Mi;
  if (hi > (i64)(j + 1) * M) hi = (i64)(j + 1) * M;
  if (hi > len) hi = len;
  if (lo > hi) lo = hi;
}
// Number of TMA tiles of micro-batch j (16-byte-aligned body only).  A stage holds one
// reduce tile (A and B halves of RESCCL_TMA_TILE bytes) or one copy tile of twice that.
// (A bulk-reduced primitive stages only the incoming operand: a whole-stage tile, as a copy.)
template <int F>
__device__ __forceinline__ i64 tile_bytes(bool bred = false) {
  return ((F & kReduce) && !bred) ? RESCCL_TMA_TILE : 2 * RESCCL_TMA_TILE;
}
template <int F>
__device__ __forceinline__ u32 mb_tiles_m(i64 M, i64 Mi, i64 len, int j, int inst, int esz, i64& lo, i64& nb,
                                          bool bred = false) {
  i64 hi;
  slice_of_m(M, Mi, len, j, inst, lo, hi);
  nb = ((hi - lo) * esz) & ~(i64)15;
  return (u32)((nb + tile_bytes<F>(bred) - 1) / tile_bytes<F>(bred));
}
template <int F>
__device__ __forceinline__ u32 mb_tiles(const KArgs& a, i64 len, int j, int inst, int esz, i64& lo, i64& nb) {
  i64 hi;
  slice_of(a, len, j, inst, lo, hi);
  nb = ((hi - lo) * esz) & ~(i64)15;
  return (u32)((nb + tile_bytes<F>() - 1) / tile_bytes<F>());
}

// TMA pipeline, leader thread: a non-blocking event loop that (1) confirms the
// readiness of the next micro-batch, (2) streams its tiles into its stages with
// cp.async.bulk, (3) stores tiles whose data is loaded (copy) or combined (reduce) to
// the local buffer and/or the peer FIFO, (4) posts a micro-batch once all its stores
// completed.  It never blocks on a remote condition while it holds unposted work, so
// the pipeline adds no wait edge beyond those of the blocking model (deadlock freedom
// carries over from the plan check).
template <class T, int OP, int F, bool BRED>
__device__ __noinline__ bool pipe_leader(Lane& L, const PrimDesc& d, const PrimPtrs& p) {
#if RESCCL_PHASE
  L.t_pro = ph_now();
#endif
  const KArgs& a = *L.a;
  // Everything the loop reads per tile lives in registers: the lane, the arguments and
  // the pointers are memory-resident (their addresses are taken), and every asm
  // statement below clobbers memory, so field accesses would reload them each time.
  const u32 Lfull = L.full, Lcomp = L.comp, Lpool = L.pool, Lqprog = L.qprog, Lqdesc = L.qdesc, Lwant = L.want;
  const int Linst = L.inst, Lbar = L.bar;
  const u32 Lring0 = L.ring0;
  u32 Lcpar = L.cpar;
  const i64 aM = a.M, aMi = a.Mi, plen = p.len;
  const char* const pA = p.A;
  const char* const pR = p.R;
  char* const pQ = p.Q;
  char* const pD1 = p.D1;
  char* const pin = p.in_data;
  char* const pout = p.out_data;
  const u32 P = RESCCL_POOL;  // slots of the per-tile register records (>= stages held)
  constexpr bool bred = BRED;  // (a template parameter: the per-tile loop stays branch-free)
  const i64 TB = tile_bytes<F>(bred);
  const int nmb = a.n_mb;
  const u32 k0 = L.tseq;
  const u32 sbase = L.stage;
  const u64 mb_base = a.mb_base;
  int rj = 0;                 // micro-batches whose readiness is confirmed
  int lj = 0;                 // load cursor (micro-batch, tile)
  u32 lt = 0;
  u32 issued = 0, stored = 0, released = 0;  // tiles (released: stage read out by its store)
  // per in-flight tile (slot = tile % P), kept in registers: its stage (4 bits) and the
  // parities of its full / comp barrier phases (1 bit each)
  u64 hs = 0;
  u32 hf = 0, hc = 0;
#define RESCCL_HS(slot) ((u32)(hs >> (4 * (slot))) & 15u)
#if RESCCL_RING
  const u32 eR = RESCCL_TMA_STAGES;
#else
  u32 emask = 0, eR = 0;      // the epoch's stages (bit mask, count)
  u64 ering = 0;              // their ids in ascending order, 4 bits each
  u32 epar = 0, ecpar = 0;    // base full / comp phase parity per ring position
  u32 li = 0, lu = 0;         // ring position / use parity of the next load
  bool wanting = false, shrink = false;
  u32 published = 0;          // tiles announced to the combine warps
  u32 ebase = 0;              // first tile of the epoch
  const u32 want_self = Lwant + 4 * (Lbar - 1), want_other = Lwant + 4 * (2 - Lbar);
#endif
  int sj = 0;                 // store cursor
  u32 st = 0;
  int pj = 0;                 // next micro-batch to post
  i64 lo_l = 0, nb_l = 0, lo_s = 0, nb_s = 0, lo_p = 0, nb_p = 0;
  u32 T_l = mb_tiles_m<F>(aM, aMi, plen, 0, Linst, T::kSize, lo_l, nb_l, bred);
  u32 T_s = T_l;
  lo_s = lo_l;
  nb_s = nb_l;
  u32 T_p = T_l;
  lo_p = lo_l;
  nb_p = nb_l;
  u32 gp_end = T_l;           // tiles through micro-batch pj
  u64 t_idle = 0, t_wd = 0;  // idle interval start (trace), watchdog start
  u32 spins = 0;
  const u64 pol_first = policy_evict_first();
  const u64 pol_last = policy_evict_last();
  int pf = 0;                 // next micro-batch whose local slice gets an L2 prefetch
  int wp = 0;                 // push receiver (drecv_d): micro-batches posted "writable"
#if RESCCL_PHASE
  // phase records: t0 previous post (or entry), t1 micro-batch ready (dependencies, flag,
  // credit), t3 every store of it complete, t4 posted
  u64 ph_rdy[8], ph_w = ph_now();
#endif
  while (pj < nmb) {
    bool prog = false;
    if (Kind<F>::push_recv) {  // post "writable" as far ahead as the dependencies allow
#if RESCCL_LOOKAHEAD
      for (int n2; wp < nmb; wp = n2) {  // through the lane's writable cursor (R30)
        lookahead(L);
        n2 = writable_posted(L, nmb);
        if (n2 <= wp) break;
        prog = true;
      }
#else
      while (wp < nmb) {
        bool ok = true;
        for (int k = 0; k < d.ndeps && ok; ++k)
          ok = dep_ready(L, d, k, wp);
        if (!ok) break;
        post_writable<F>(a, d, p, wp);
        ++wp;
        prog = true;
      }
#endif
    }
#if RESCCL_PREFETCH
    // (0) keep the local operand of the next RESCCL_PREFETCH micro-batches streaming into L2
    if (pA && (F & (kReduce | kRecv)) != kRecv) {
      while (pf < nmb && pf <= lj + RESCCL_PREFETCH) {
        i64 lo_f, nb_f;
        mb_tiles_m<F>(aM, aMi, plen, pf, Linst, T::kSize, lo_f, nb_f);
        if (nb_f > 0) l2_prefetch(pA + lo_f * T::kSize, (u32)nb_f);
        ++pf;
      }
    }
#endif
    // (1) readiness of the micro-batch the load cursor needs
    if (rj < nmb && rj == lj && (!Kind<F>::push_recv || rj < wp) && mb_ready<F>(L, d, p, rj)) {
      fence_proxy_async();  // generic-proxy data (acquired) -> async-proxy reads
#if RESCCL_PHASE
      ph_rdy[rj & 7] = ph_now();
#endif
      ++rj;
      prog = true;
    }
    // (2) loads
    while (lj < rj) {
      if (lt >= T_l) {
        ++lj;
        lt = 0;
        if (lj < nmb) T_l = mb_tiles_m<F>(aM, aMi, plen, lj, Linst, T::kSize, lo_l, nb_l, bred);
        continue;
      }
#if !RESCCL_RING
      if (shrink) break;
      if (eR == 0) {  // start an epoch: take the free stages
        u32 m = atoms_and(Lpool, 0u);
        const u32 cap = lds_u32(want_other) ? (P / 2 < RESCCL_POOL_CAP ? P / 2 : RESCCL_POOL_CAP)
                                            : (u32)RESCCL_POOL_CAP;
        u32 keep = 0;
        for (u32 n = 0; m && n < cap; ++n) {
          const u32 b = m & (0u - m);
          keep |= b;
          m &= ~b;
        }
        if (m) atoms_or(Lpool, m);  // over the cap: give back
        if (!keep) {
          if (!wanting) sts_u32(want_self, 1u);
          wanting = true;
          break;  // the other lane holds the pool: its tiles drain by themselves
        }
        if (wanting) sts_u32(want_self, 0u);
        wanting = false;
        emask = keep;
        eR = (u32)__popc(keep);
        ering = 0;
        epar = 0;
        ecpar = 0;
        for (u32 i = 0, mm = keep; mm; ++i) {
          const u32 s = (u32)(__ffs(mm) - 1);
          mm &= mm - 1;
          ering |= (u64)s << (4 * i);
          epar |= mbar_phase(Lfull + 8 * s) << i;
          ecpar |= mbar_phase(Lcomp + 8 * s) << i;
        }
        li = 0;
        lu = 0;
        ebase = k0 + issued;
        // the combine warps map this epoch's tiles through (first tile, stages, parities);
        // the announcements carry the first tile too, so a reader validates the
        // descriptor against them (no fence)
        if (F & kReduce) sts_u64(Lqdesc, (u64)ebase | ((u64)emask << 32) | ((u64)epar << 48));
      }
#endif
      if (issued - released >= eR) {  // the tile eR back still holds the stage we need next
        if (stored > released && (stored - released >= (u32)RESCCL_STORE_LAG || issued == stored)) {
          const u32 keep = stored - released - 1 < 15 ? stored - released - 1 : 15;
          tma_wait_read_n(keep);
          released = stored - keep;
        }
        if (issued - released >= eR) break;
      }
      const u32 k = k0 + issued;
      const u32 slot = issued % P;
#if RESCCL_RING
      const u32 s = Lring0 + k % RESCCL_TMA_STAGES;
      const u32 fpar = (k / RESCCL_TMA_STAGES) & 1;
      if ((F & kReduce) && !bred) {
        const u32 rb = 1u << (k % RESCCL_TMA_STAGES);
        hc = (hc & ~(1u << slot)) | (((Lcpar & rb) ? 1u : 0u) << slot);
        Lcpar ^= rb;
      }
#else
      const u32 s = (u32)(ering >> (4 * li)) & 15u;
      const u32 fpar = ((epar >> li) & 1u) ^ lu;
      if (F & kReduce) hc = (hc & ~(1u << slot)) | ((((ecpar >> li) & 1u) ^ lu) << slot);
      if (++li == eR) {
        li = 0;
        lu ^= 1u;
      }
      // every 32 tiles: the other lane waits for stages while we hold more than half
      if (eR > P / 2 && (issued & 31) == 31 && lds_u32(want_other)) shrink = true;
#endif
      hs = (hs & ~(15ull << (4 * slot))) | ((u64)s << (4 * slot));
      hf = (hf & ~(1u << slot)) | (fpar << slot);
      const i64 off = (i64)lt * TB;
      const u32 nb = (u32)((nb_l - off) < TB ? (nb_l - off) : TB);
      const u32 sa = sbase + s * 2 * (u32)RESCCL_TMA_TILE;
      if (F & kReduce) {
        const u64 in_seq = (u64)d.in_n * mb_base + (u64)d.in_pos * nmb + lj;
        const char* bsrc = (F & kDirect) ? pR + lo_l * T::kSize + off
                                         : pin + (in_seq % RESCCL_K) * RESCCL_SLOT + off;
        if (bred) {  // incoming tile only; the local operand is added in L2 by the store
          mbar_expect_tx(Lfull + 8 * s, nb);
          tma_load(sa, bsrc, nb, Lfull + 8 * s, pol_first);
        } else {
          mbar_expect_tx(Lfull + 8 * s, 2 * nb);
          tma_load(sa, pA + lo_l * T::kSize + off, nb, Lfull + 8 * s, pol_first);
          tma_load(sa + (u32)RESCCL_TMA_TILE, bsrc, nb, Lfull + 8 * s, pol_first);
        }
      } else {
        const char* src;
        if (Kind<F>::has_b) {  // staged receive: the FIFO slot
          const u64 in_seq = (u64)d.in_n * mb_base + (u64)d.in_pos * nmb + lj;
          src = pin + (in_seq % RESCCL_K) * RESCCL_SLOT + off;
        } else {               // send / pushed payload forwarded: our location
          src = pA + lo_l * T::kSize + off;
        }
        mbar_expect_tx(Lfull + 8 * s, nb);
        tma_load(sa, src, nb, Lfull + 8 * s, pol_first);
      }
      (void)k;
      ++issued;
      ++lt;
      prog = true;
    }
#if !RESCCL_RING
    if ((F & kReduce) && !bred && published != issued) {  // one word per batch of issued tiles
      sts_u64(Lqprog, ((u64)ebase << 32) | (u64)(k0 + issued));
      published = issued;
    }
#endif
    // (3) stores
    while (stored < issued) {
      const u32 slot = stored % P;
      const u32 s = RESCCL_HS(slot);
      const bool ok = ((F & kReduce) && !bred) ? mbar_test(Lcomp + 8 * s, (hc >> slot) & 1)
                                               : mbar_test(Lfull + 8 * s, (hf >> slot) & 1);
      if (!ok) break;
      while (st >= T_s) {
        ++sj;
        st = 0;
        T_s = mb_tiles_m<F>(aM, aMi, plen, sj, Linst, T::kSize, lo_s, nb_s, bred);
      }
      const i64 off = (i64)st * TB;
      const u32 nb = (u32)((nb_s - off) < TB ? (nb_s - off) : TB);
      const u32 sa = sbase + s * 2 * (u32)RESCCL_TMA_TILE;
      if ((F & kStore) && pD1) {
        if ((F & kReduce) && bred) tma_reduce<T, OP>(pD1 + lo_s * T::kSize + off, sa, nb, pol_first);
        else tma_store(pD1 + lo_s * T::kSize + off, sa, nb, pol_first);
      }
      if (Kind<F>::send_data) {
        if (F & kDirect) {
          tma_store(pQ + lo_s * T::kSize + off, sa, nb, pol_first);
        } else {
          const u64 out_seq = (u64)d.out_n * mb_base + (u64)d.out_pos * nmb + sj;
          tma_store(pout + (out_seq % RESCCL_K) * RESCCL_SLOT + off, sa, nb, pol_last);
        }
      }
      tma_commit();
      ++stored;
      ++st;
      prog = true;
    }
    // (4) post
    if (pj < rj && stored >= gp_end) {
      tma_wait_n(stored - gp_end);
      if (released < gp_end) released = gp_end;  // written out
      // unaligned tail (< 16 bytes) of this micro-batch: scalar, by the leader
      i64 lo_h, hi_h;
      slice_of_m(aM, aMi, plen, pj, Linst, lo_h, hi_h);
      const i64 e0 = lo_h + nb_p / T::kSize;
      if (e0 < hi_h) {
        const u64 in_seq = (u64)d.in_n * mb_base + (u64)d.in_pos * nmb + pj;
        const u64 out_seq = (u64)d.out_n * mb_base + (u64)d.out_pos * nmb + pj;
        const char* Bj = Kind<F>::has_b ? ((F & kDirect) ? pR + e0 * T::kSize
                                                         : pin + (in_seq % RESCCL_K) * RESCCL_SLOT + nb_p)
                                        : nullptr;
        char* D2j = Kind<F>::send_data ? ((F & kDirect) ? pQ + e0 * T::kSize
                                                        : pout + (out_seq % RESCCL_K) * RESCCL_SLOT + nb_p)
                                       : nullptr;
        for (i64 e = 0; e < hi_h - e0; ++e)
          elem_move<T, OP>(Kind<F>::mf, pA ? pA + e0 * T::kSize : nullptr, Bj,
                           pD1 ? pD1 + e0 * T::kSize : nullptr, D2j, e);
      }
      fence_proxy_async();
#if RESCCL_PHASE
      const u64 ph3 = ph_now();
#endif
      post_mb<F>(a, d, p, pj);
#if RESCCL_PHASE
      ph_rec(L, PhPipe, pj, ph_w, ph_rdy[pj & 7], pj == 0 ? L.t_run : 0, ph3, ph_now());
      ph_w = ph_now();
#endif
      ++pj;
#if RESCCL_EARLY_EXIT
      if (pj == nmb) break;  // all posted: the code after the loop returns the stages
#else
      if (pj < nmb)
#endif
      {
        T_p = mb_tiles_m<F>(aM, aMi, plen, pj, Linst, T::kSize, lo_p, nb_p, bred);
        gp_end += T_p;
      }
      prog = true;
    }
#if !RESCCL_RING
    // (5) end the epoch once everything loaded is stored and no ready work is left (or
    // when shrinking), after the stores have read their stages out
    if (eR && stored == issued && (lj == rj || shrink)) {
      if (stored > released) {
        tma_wait_read_n(0);
        released = stored;
      }
      atoms_or(Lpool, emask);
      eR = 0;
      emask = 0;
      shrink = false;
    }
#endif
    if (prog) {
      idle_off(L, t_idle);
      spins = 0;
    } else {
      // idle = busy-waiting with no data of this lane in flight (tiles outstanding are the
      // data path working, not a wait for a peer)
      if (stored == issued) idle_on(L, t_idle);
      else idle_off(L, t_idle);
#if RESCCL_LOOKAHEAD
      if (stored == issued && (spins & 3) == 0 && L.wa_c < L.wa_n) lookahead(L);  // only while data-idle
                                                                                 // (register tests first)
#endif
      if (stored < issued) {
        // idle with a tile outstanding: sleep on the oldest one's barrier (it is the next
        // event the store step needs) instead of polling
        const u32 slot = stored % P;
        const u32 s = RESCCL_HS(slot);
        if ((F & kReduce) && !bred) (void)mbar_try(Lcomp + 8 * s, (hc >> slot) & 1);
        else (void)mbar_try(Lfull + 8 * s, (hf >> slot) & 1);
        ++spins;
      } else if (++spins > 32) {
        nanosleep_(20);
      }
      if ((spins & 255) == 0) {
        const u64 now = globaltimer();
        if (t_wd == 0) t_wd = now;
        else if (now - t_wd > a.timeout_ns) {
          atomicCAS(a.err, 0, kErrTimeout);
          *L.abort_flag = 1;
          return false;
        }
      }
    }
    if (prog) t_wd = 0;
  }
  if (stored > released) {  // (all posted: every store has completed)
    tma_wait_read_n(0);
    released = stored;
  }
#if !RESCCL_RING
  if (eR) atoms_or(Lpool, emask);
  if (wanting) sts_u32(want_self, 0u);
#endif
#undef RESCCL_HS
  idle_off(L, t_idle);
  L.tseq = k0 + issued;
  L.cpar = Lcpar;
#if RESCCL_PHASE
  L.t_end = ph_now();
#endif
  return true;
}

// TMA pipeline, combine warps (reduce primitives): tile k of the lane's stream is
// combined in shared memory as soon as its A and B tiles land.
template <class T, int OP, int F>
__device__ __noinline__ bool pipe_compute(Lane& L, const PrimDesc& d, const PrimPtrs& p, int ctid, int nct) {
  const KArgs& a = *L.a;
  const i64 TB = RESCCL_TMA_TILE;  // reduce tiles only
  const u32 Lfull = L.full, Lcomp = L.comp, Lstage = L.stage, Lqprog = L.qprog, Lqdesc = L.qdesc, Lring0 = L.ring0;
  const int Linst = L.inst, nmb = a.n_mb, Lbar = L.bar;
  const i64 aM = a.M, aMi = a.Mi, plen = p.len;
  volatile int* const abort_flag = L.abort_flag;
  u32 k = L.tseq;
  if (bulk_reduce_prim<T, OP, F>(p.A, p.D1)) {  // the leader adds in L2: only keep the tile count
    for (int j = 0; j < nmb; ++j) {
      i64 lo, nbj;
      k += mb_tiles_m<F>(aM, aMi, plen, j, Linst, T::kSize, lo, nbj, true);
    }
    L.tseq = k;
    return true;
  }
#if !RESCCL_RING
  u32 cbase = 0xFFFFFFFFu, cmask = 0, cpar = 0, cR = 1, ci = 0, cu = 0;  // cached epoch, position of k
#endif
  for (int j = 0; j < nmb; ++j) {
    i64 lo, nbj;
    const u32 ntl = mb_tiles_m<F>(aM, aMi, plen, j, Linst, T::kSize, lo, nbj);
    for (u32 t = 0; t < ntl; ++t, ++k) {
      const i64 off = (i64)t * TB;
      const int nb = (int)((nbj - off) < TB ? (nbj - off) : TB);
      u32 spins = 0;
#if RESCCL_RING
      // stage and phase follow from k (the leader cannot re-arm the stage for tile k + S
      // before every combine warp arrived for tile k: no parity ABA)
      const u32 s = Lring0 + k % RESCCL_TMA_STAGES;
      const u32 par = (k / RESCCL_TMA_STAGES) & 1;
#else
      // wait until the leader announced tile k (announcement = epoch's first tile << 32 |
      // tiles issued), then map it through that epoch: the epoch holding tile k cannot end
      // before this warp combined it, so the announcing epoch is k's
      u64 w;
#if RESCCL_CPOLL
      // one polling warp; the others sleep on the combine warps' named barrier instead of
      // queueing shared-memory loads behind the TMA traffic
      if (ctid < 32) {
        while ((int)((u32)lds_u64(Lqprog) - k) <= 0) {
          if (++spins > 16) nanosleep_(20);
          if ((spins & 1023) == 0 && *abort_flag) break;
        }
      }
      asm volatile("barrier.sync %0, %1;" ::"r"(Lbar + 2), "r"(nct) : "memory");
      if (*abort_flag) return false;
      w = lds_u64(Lqprog);
#else
      while ((int)((u32)(w = lds_u64(Lqprog)) - k) <= 0) {
        if (++spins > 16) nanosleep_(20);
        if ((spins & 1023) == 0 && *abort_flag) return false;
      }
#endif
      const u32 eb = (u32)(w >> 32);
      if (eb != cbase) {  // a new epoch: its descriptor (validated by its first tile)
        u64 dsc;
        while ((u32)(dsc = lds_u64(Lqdesc)) != eb) {
        }
        cbase = eb;
        cmask = (u32)(dsc >> 32) & 0xFFFFu;
        cpar = (u32)(dsc >> 48);
        cR = (u32)__popc(cmask);
        ci = (k - eb) % cR;
        cu = ((k - eb) / cR) & 1u;
      }
      const u32 s = nth_bit(cmask, ci);
      const u32 par = ((cpar >> ci) & 1u) ^ cu;
      if (++ci == cR) {
        ci = 0;
        cu ^= 1u;
      }
#endif
      while (!mbar_try(Lfull + 8 * s, par)) {  // (stage s is held for tile k: no parity ABA)
        if ((++spins & 63) == 0 && *abort_flag) return false;
      }
      const u32 sa = Lstage + s * 2 * (u32)TB;
      for (int i2 = ctid; i2 < nb / 16; i2 += nct)
        sts_v4(sa + 16 * i2, combine_v<T, OP>(lds_v4(sa + 16 * i2), lds_v4(sa + (u32)TB + 16 * i2)));
      fence_proxy_async_smem();
      __syncwarp();
      if ((threadIdx.x & 31) == 0) mbar_arrive(Lcomp + 8 * s);
    }
  }
  L.tseq = k;
  return true;
}

// Direct-mode primitives that move no data (leader only): a pull-send posts "readable"
// for each micro-batch once its dependencies hold; a push-receive posts "writable"
// (credit) as soon as its dependencies hold -- running ahead of the payloads -- and
// completes a micro-batch when the sender's "written" flag arrives (drecv_p then also
// posts "readable" for the next hop, which pulls from our location).
template <int F>
__device__ __noinline__ bool run_flags(Lane& L, const PrimDesc& d, const PrimPtrs& p) {
#if RESCCL_PHASE
  L.t_pro = ph_now();
#endif
  const KArgs& a = *L.a;
  const int nmb = a.n_mb;
  const u64 mb_base = a.mb_base;
  constexpr bool recv = F & kRecv;
  int wp = 0, dj = 0;  // posted (readable / writable) / completed micro-batches
  u64 t_idle = 0, t_wd = 0;  // idle interval start (trace), watchdog start
  u32 spins = 0;
  // phase records: t0 start of the wait, t1 dependencies met (readable / writable
  // posted right after), t2 the peer's "written" flag seen (push receive), t4 posted
  u64 ph_w = ph_now(), ph_dep[4] = {0, 0, 0, 0};
  while (recv ? dj < nmb : wp < nmb) {
    bool prog = false;
#if RESCCL_LOOKAHEAD
    if (recv && wp < nmb) {  // writable credits go through the lane's cursor (R30)
      lookahead(L);
      const int n2 = writable_posted(L, nmb);
      if (n2 > wp) prog = true;
      for (; wp < n2; ++wp) ph_dep[wp & 3] = ph_now();
    }
    if (!recv && wp < nmb) {
#else
    if (wp < nmb) {
#endif
      bool ok = true;
      for (int k = 0; k < d.ndeps && ok; ++k)
        ok = dep_seen(L, d, k, wp);  // (the fence.acq_rel below acquires it)
      if (ok) {
        const u64 ph1 = ph_now();
        fence_release();
        if (!recv) {
          const u64 out_seq = (u64)d.out_n * mb_base + (u64)d.out_pos * nmb + wp;
          st_relaxed(p.out_flag + (out_seq % RESCCL_K), out_seq + 1);
          ph_rec(L, PhFlags, wp, ph_w, ph1, 0, 0, ph_now());
          ph_w = ph_now();
        } else {
          const u64 in_seq = (u64)d.in_n * mb_base + (u64)d.in_pos * nmb + wp;
          st_relaxed(p.in_cred, in_seq + 1);
          ph_dep[wp & 3] = ph1;
        }
        ++wp;
        prog = true;
      }
    }
    if (recv && dj < wp) {
      const u64 in_seq = (u64)d.in_n * mb_base + (u64)d.in_pos * nmb + dj;
      if (ld_relaxed(p.in_flag + (in_seq % RESCCL_K)) >= in_seq + 1) {  // (acquired by the fence below)
        const u64 ph2 = ph_now();
        fence_release();
        if (F & kSend) {  // drecv_p: the payload is in our location -> readable for the next hop
          const u64 out_seq = (u64)d.out_n * mb_base + (u64)d.out_pos * nmb + dj;
          st_relaxed(p.out_flag + (out_seq % RESCCL_K), out_seq + 1);
        }
        if (d.ctr >= 0) st_relaxed(p.ctr, mb_base + dj + 1);
        ph_rec(L, PhFlags, dj, ph_w, ph_dep[dj & 3], ph2, 0, ph_now());
        ph_w = ph_now();
        ++dj;
        prog = true;
      }
    }
    if (prog) {
      idle_off(L, t_idle);
      spins = 0;
      t_wd = 0;
    } else {
      idle_on(L, t_idle);
#if RESCCL_LOOKAHEAD
      if (L.wa_c < L.wa_n && (spins & 7) == 7) lookahead(L);  // rate-limited: the flag poll first
#endif
      if (++spins > 32) nanosleep_(20);
      if ((spins & 255) == 0) {
        const u64 now = globaltimer();
        if (t_wd == 0) t_wd = now;
        else if (now - t_wd > a.timeout_ns) {
          atomicCAS(a.err, 0, kErrTimeout);
          *L.abort_flag = 1;
          return false;
        }
      }
    }
  }
  idle_off(L, t_idle);
#if RESCCL_PHASE
  L.t_end = ph_now();
#endif
  return true;
}

// A run of consecutive dependency-free pull-sends in one lane (e.g. the full mesh's seven
// "readable" posts of its sendbuf chunks, PAPER Fig. 16): a pull-send without dependencies
// publishes a location no primitive of this kernel writes, so nothing has to be waited for;
// run one by one, each cost a primitive switch and a fence (~1.3 us, §5.12c) and the last
// peer to be told waited ~9 us.  One release fence, then every flag in program order (each
// link's positions still increase, R26).  Leader only; the other threads have nothing to do.
template <int F>
__device__ __noinline__ bool run_post_group(Lane& L, const PrimDesc* descs, const int* idx, int n) {
#if RESCCL_PHASE
  L.t_run = ph_now();
#endif
  if (L.tid != 0) return true;
  const KArgs& a = *L.a;
  const int nmb = a.n_mb;
  const u64 ph_w = ph_now();
  fence_rel();
  for (int i = 0; i < n; ++i) {
    const PrimDesc& d = descs[idx[i]];
    u64* const out_flag = at(a.arena[d.out_peer], d.out_flag + (i64)L.inst * RESCCL_FLAGSTRIDE);
    for (int j = 0; j < nmb; ++j) {
      const u64 out_seq = (u64)d.out_n * a.mb_base + (u64)d.out_pos * nmb + j;
      st_relaxed(out_flag + (out_seq % RESCCL_K), out_seq + 1);
#if RESCCL_PHASE
      L.pidx = idx[i];
      ph_rec(L, PhFlags, j, ph_w, ph_w, 0, 0, ph_now());
#endif
    }
  }
  return true;
}

template <class T, int OP, int F>
__device__ __noinline__ bool run(Lane& L, const PrimDesc& d) {
#if RESCCL_PHASE
  L.t_run = ph_now();
#endif
  const KArgs& a = *L.a;
  const int c = d.chunk;
  PrimPtrs p;
  p.len = chunk_len<RESCCL_COLL>(a, c);
  p.A = nullptr;
  p.D1 = nullptr;
  if (d.src_buf != BufNone && ((F & kCopy) || (F & kReduce) || !Kind<F>::has_b))
    p.A = buf_ptr(a, L.rank, d.src_buf) + chunk_off<RESCCL_COLL>(d.src_buf, c, a.C) * T::kSize;
  if ((F & kCopy) || (F & kStore))
    p.D1 = buf_ptr(a, L.rank, d.dst_buf) + chunk_off<RESCCL_COLL>(d.dst_buf, c, a.C) * T::kSize;
  // a send storing an unwritten output locally (AllGather's own chunk): in place the
  // output already holds it
  if ((F & kSend) && (F & kStore) && !(F & kRecv) && p.A == p.D1) p.D1 = nullptr;
  if (F & kCopy) {
    if (p.A == p.D1) return true;  // in-place: own chunk already in place
    for (int j = 0; j < a.n_mb; ++j) {
      i64 lo, hi;
      slice_of(a, p.len, j, L.inst, lo, hi);
      move<T, OP, kCopy, 4>(hi - lo, p.A + lo * T::kSize, nullptr, p.D1 + lo * T::kSize, nullptr, L.tid, L.nthreads);
    }
    return true;
  }
  p.in_data = L.self + d.in_data + (i64)L.inst * RESCCL_K * RESCCL_SLOT;
  p.in_flag = at(L.self, d.in_flag + (i64)L.inst * RESCCL_FLAGSTRIDE);
  p.in_cred = (F & kRecv) ? at(a.arena[d.in_peer], d.in_cred + (i64)L.inst * 128) : nullptr;
  char* peer = (F & kSend) ? a.arena[d.out_peer] : nullptr;
  p.out_data = (F & kSend) ? peer + d.out_data + (i64)L.inst * RESCCL_K * RESCCL_SLOT : nullptr;
  p.out_flag = (F & kSend) ? at(peer, d.out_flag + (i64)L.inst * RESCCL_FLAGSTRIDE) : nullptr;
  p.out_cred = at(L.self, d.out_cred + (i64)L.inst * 128);
  p.ctr = at(L.self, d.ctr + (i64)L.inst * 128);
  p.R = ((F & kDirect) && (F & kPull))
            ? buf_ptr(a, d.rem_rank, d.rem_buf) + chunk_off<RESCCL_COLL>(d.rem_buf, c, a.C) * T::kSize
            : nullptr;
  p.Q = ((F & kDirect) && Kind<F>::send_data)
            ? buf_ptr(a, d.out_rank, d.out_buf) + chunk_off<RESCCL_COLL>(d.out_buf, c, a.C) * T::kSize
            : nullptr;
  // no data moved here: pull-send, push-receive (+ readable for the next hop)
  if ((F & kDirect) && !Kind<F>::has_b && !Kind<F>::send_data) return L.tid == 0 ? run_flags<F>(L, d, p) : true;
#ifndef RESCCL_TMA_MIN
#define RESCCL_TMA_MIN 32768
#endif
#if RESCCL_TMA
  // small slices are latency-bound: the register path saves two bulk-copy round trips
  const unsigned long long al =
      (unsigned long long)p.A | (unsigned long long)p.D1 | (unsigned long long)p.R | (unsigned long long)p.Q;
  if ((al & 15) == 0 && a.Mi * T::kSize >= RESCCL_TMA_MIN) {
    if (L.tid == 0)
      return bulk_reduce_prim<T, OP, F>(p.A, p.D1) ? pipe_leader<T, OP, F, RESCCL_BULKRED != 0>(L, d, p)
                                                   : pipe_leader<T, OP, F, false>(L, d, p);
    if (L.tid < 32) return true;
    if (F & kReduce) return pipe_compute<T, OP, F>(L, d, p, L.tid - 32, L.nthreads - 32);
    // combine warps only keep the lane's tile counter in step for copy primitives
    for (int j = 0; j < a.n_mb; ++j) {
      i64 lo, nb;
      L.tseq += mb_tiles<F>(a, p.len, j, L.inst, T::kSize, lo, nb);
    }
    return true;
  }
#endif
  return run_sync<T, OP, F>(L, d, p);
}

// Direct transport across processes (RESCCL_EXIT_BARRIER): peers pull from and push into
// this rank's user buffers, so this rank's kernel -- whose completion hands the buffers
// back to the caller -- must not end before every peer block is done with them.  Every
// block adds 1 to its rank's monotone done counter (release); block 0 then waits until
// each peer's counter covers this call: (epoch + 1) x that peer's block count.
__device__ __noinline__ void exit_barrier(const KArgs& a, int rank, int nranks, const int* blocks, i64 off) {
  cta_sync();
  if (threadIdx.x != 0) return;
  fence_release();
  asm volatile("red.release" RESCCL_SC ".global.add.u64 [%0], 1;" ::"l"(at(a.arena[rank], off)) : "memory");
  if (blockIdx.x != 0) return;
  const u64 t0 = globaltimer();
  for (int q = 0; q < nranks; ++q) {
    if (q == rank) continue;
    const u64 target = (a.epoch + 1) * (u64)blocks[q];
    u32 spins = 0;
    while (!ready_ge(at(a.arena[q], off), target)) {
      if (++spins > 64) nanosleep_(64);
      if ((spins & 1023) == 0 && globaltimer() - t0 > a.timeout_ns) {
        atomicCAS(a.err, 0, kErrTimeout);
        return;
      }
    }
  }
}

// ============================================================================= f3: NVLS transport
// NVLink SHARP (not in the paper, the B200 NVSwitch variant of the
// transport).  Every rank's buffer is bound into one multicast object, so a load through
// the multicast alias (multimem.ld_reduce) returns the reduction of all ranks' copies,
// computed inside the switch, and a store through it (multimem.st) lands in every rank's
// copy.  On the collective's chunk layout (R6: chunk c belongs to rank c) the schedule is
//   mred(r): <r,c=r> := (+)_k <k,r>     (ReduceScatter; one multimem.ld_reduce per granule)
//   mcast(r): <k,r>  := <r,r>  for all k (AllGather; one multimem.st per granule)
// and AllReduce = mred then mcast of each rank's own chunk.  mcast(r)
// depends only on mred(r) of the same granule in the same thread, so no barrier sits
// between the phases; an entry barrier orders every rank's earlier writes of its send
// buffer before anyone's multimem loads, and an exit barrier keeps a rank's kernel alive
// until every peer's multicast stores into its receive buffer have landed.
// Granules are 16 bytes (v4) when every address is 16-byte aligned, else 4 bytes; the
// host only routes calls whose per-rank blocks are whole 4-byte granules here (2-byte
// dtypes: even counts) and f32 max/min, which multimem.ld_reduce lacks, elsewhere.
struct NvlsArgs {
  char* mc_send;         // multicast alias of sendbuf (AR/RS) -- null for AG
  char* mc_recv;         // multicast alias of recvbuf (AR/AG) -- null for RS
  const char* uc_send;   // this rank's sendbuf (AG source)
  char* uc_recv;         // this rank's recvbuf (RS destination)
  u32* mc_flags;         // multicast alias of the window's barrier words [entry, exit]
  u32* uc_flags;         // this rank's copy of them
  i64 lo_bytes;          // this rank's byte range [lo, hi) of the AR buffer / RS,AG block
  i64 hi_bytes;
  u32 target;            // barrier arrivals on this window once this call's have landed
  int nranks;
  int vec;               // 1: 16-byte granules, 0: 4-byte granules
  int* err;
  u64 timeout_ns;
};

template <class T, int OP>
__device__ __forceinline__ void mm_ldred4(const char* mc, u32 (&v)[4]);
template <class T, int OP>
__device__ __forceinline__ u32 mm_ldred1(const char* mc);

#define RESCCL_MM_V4(SUF)                                                                   \
  asm volatile("multimem.ld_reduce.relaxed.sys.global." SUF " {%0,%1,%2,%3}, [%4];"          \
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "l"(mc) : "memory")
#define RESCCL_MM_S4(SUF)                                                                   \
  asm volatile("multimem.ld_reduce.relaxed.sys.global." SUF " %0, [%1];" : "=r"(x) : "l"(mc) : "memory")
#define RESCCL_MM_INT4(SUF)                                                                 \
  for (int j = 0; j < 4; ++j)                                                               \
    asm volatile("multimem.ld_reduce.relaxed.sys.global." SUF " %0, [%1];"                  \
                 : "=r"(v[j]) : "l"(mc + 4 * j) : "memory")

// bf16 / f16 sums accumulate in fp32 inside the switch and round once (acc::f32)
template <> __device__ __forceinline__ void mm_ldred4<TBF16, OpSum>(const char* mc, u32 (&v)[4]) { RESCCL_MM_V4("add.acc::f32.v4.bf16x2"); }
template <> __device__ __forceinline__ void mm_ldred4<TBF16, OpMax>(const char* mc, u32 (&v)[4]) { RESCCL_MM_V4("max.v4.bf16x2"); }
template <> __device__ __forceinline__ void mm_ldred4<TBF16, OpMin>(const char* mc, u32 (&v)[4]) { RESCCL_MM_V4("min.v4.bf16x2"); }
template <> __device__ __forceinline__ void mm_ldred4<TF16, OpSum>(const char* mc, u32 (&v)[4]) { RESCCL_MM_V4("add.acc::f32.v4.f16x2"); }
template <> __device__ __forceinline__ void mm_ldred4<TF16, OpMax>(const char* mc, u32 (&v)[4]) { RESCCL_MM_V4("max.v4.f16x2"); }
template <> __device__ __forceinline__ void mm_ldred4<TF16, OpMin>(const char* mc, u32 (&v)[4]) { RESCCL_MM_V4("min.v4.f16x2"); }
template <> __device__ __forceinline__ void mm_ldred4<TF32, OpSum>(const char* mc, u32 (&v)[4]) { RESCCL_MM_V4("add.v4.f32"); }
template <> __device__ __forceinline__ void mm_ldred4<TI32, OpSum>(const char* mc, u32 (&v)[4]) { RESCCL_MM_INT4("add.u32"); }
template <> __device__ __forceinline__ void mm_ldred4<TI32, OpMax>(const char* mc, u32 (&v)[4]) { RESCCL_MM_INT4("max.s32"); }
template <> __device__ __forceinline__ void mm_ldred4<TI32, OpMin>(const char* mc, u32 (&v)[4]) { RESCCL_MM_INT4("min.s32"); }
template <> __device__ __forceinline__ u32 mm_ldred1<TBF16, OpSum>(const char* mc) { u32 x; RESCCL_MM_S4("add.acc::f32.bf16x2"); return x; }
template <> __device__ __forceinline__ u32 mm_ldred1<TBF16, OpMax>(const char* mc) { u32 x; RESCCL_MM_S4("max.bf16x2"); return x; }
template <> __device__ __forceinline__ u32 mm_ldred1<TBF16, OpMin>(const char* mc) { u32 x; RESCCL_MM_S4("min.bf16x2"); return x; }
template <> __device__ __forceinline__ u32 mm_ldred1<TF16, OpSum>(const char* mc) { u32 x; RESCCL_MM_S4("add.acc::f32.f16x2"); return x; }
template <> __device__ __forceinline__ u32 mm_ldred1<TF16, OpMax>(const char* mc) { u32 x; RESCCL_MM_S4("max.f16x2"); return x; }
template <> __device__ __forceinline__ u32 mm_ldred1<TF16, OpMin>(const char* mc) { u32 x; RESCCL_MM_S4("min.f16x2"); return x; }
template <> __device__ __forceinline__ u32 mm_ldred1<TF32, OpSum>(const char* mc) { u32 x; RESCCL_MM_S4("add.f32"); return x; }
template <> __device__ __forceinline__ u32 mm_ldred1<TI32, OpSum>(const char* mc) { u32 x; RESCCL_MM_S4("add.u32"); return x; }
template <> __device__ __forceinline__ u32 mm_ldred1<TI32, OpMax>(const char* mc) { u32 x; RESCCL_MM_S4("max.s32"); return x; }
template <> __device__ __forceinline__ u32 mm_ldred1<TI32, OpMin>(const char* mc) { u32 x; RESCCL_MM_S4("min.s32"); return x; }
// f32 max/min: multimem.ld_reduce has no such form; the host never routes them here
template <> __device__ __forceinline__ void mm_ldred4<TF32, OpMax>(const char*, u32 (&v)[4]) { v[0] = v[1] = v[2] = v[3] = 0; __trap(); }
template <> __device__ __forceinline__ void mm_ldred4<TF32, OpMin>(const char*, u32 (&v)[4]) { v[0] = v[1] = v[2] = v[3] = 0; __trap(); }
template <> __device__ __forceinline__ u32 mm_ldred1<TF32, OpMax>(const char*) { __trap(); return 0; }
template <> __device__ __forceinline__ u32 mm_ldred1<TF32, OpMin>(const char*) { __trap(); return 0; }
#undef RESCCL_MM_V4
#undef RESCCL_MM_S4
#undef RESCCL_MM_INT4

__device__ __forceinline__ void mm_st4(char* mc, const u32 (&v)[4]) {
  asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(mc), "r"(v[0]), "r"(v[1]),
               "r"(v[2]), "r"(v[3])
               : "memory");
}
__device__ __forceinline__ void mm_st1(char* mc, u32 v) {
  asm volatile("multimem.st.relaxed.sys.global.b32 [%0], %1;" ::"l"(mc), "r"(v) : "memory");
}

// Grid-wide NVLS barrier on barrier word w: every block of every rank adds 1 through the
// multicast alias (release), then waits until its own copy shows all arrivals up to this
// call's: a.target = (nranks x grid) summed over the window's calls so far, this one
// included (the host keeps the sum; u32, compared wrap-safe).
__device__ __forceinline__ void nvls_barrier(const NvlsArgs& a, int w) {
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("fence.proxy.alias;" ::: "memory");
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    asm volatile("multimem.red.release.sys.global.add.u32 [%0], 1;" ::"l"(a.mc_flags + w) : "memory");
    const u32 target = a.target;
    const u64 t0 = globaltimer();
    u32 spins = 0;
    for (;;) {
      u32 x;
      asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(x) : "l"(a.uc_flags + w) : "memory");
      if ((int)(x - target) >= 0) break;  // wrap-safe
      if (++spins > 64) nanosleep_(64);
      if ((spins & 1023) == 0 && globaltimer() - t0 > a.timeout_ns) {
        atomicCAS(a.err, 0, kErrTimeout);
        break;
      }
    }
    asm volatile("fence.proxy.alias;" ::: "memory");
  }
  __syncthreads();
}

// One span of granules of G bytes (16: v4, 4: scalar), grid-strided with U granules in
// flight per thread.  coll: CollAllReduce (mred + mcast), CollReduceScatter (mred ->
// local), CollAllGather (local -> mcast).  Offsets are byte offsets into the collective's
// buffer; AR/RS read mc_send + off, AR/AG write mc_recv + off, RS writes
// uc_recv + (off - lo), AG reads uc_send + (off - lo).
template <class T, int OP, int COLL, int G>
__device__ __forceinline__ void nvls_span(const NvlsArgs& a, i64 from, i64 to) {
  const i64 tid = (i64)blockIdx.x * blockDim.x + threadIdx.x;
  const i64 nth = (i64)gridDim.x * blockDim.x;
  const i64 lo = a.lo_bytes;
  const i64 n = (to - from) / G;
  constexpr int U = 4;
  for (i64 base = tid; base < n; base += nth * U) {
    u32 v[U][4];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const i64 k = base + (i64)u * nth;
      if (k < n) {
        const i64 off = from + k * G;
        if (COLL == CollAllGather) {
          if (G == 16) {
            const uint4 w = *reinterpret_cast<const uint4*>(a.uc_send + (off - lo));
            v[u][0] = w.x; v[u][1] = w.y; v[u][2] = w.z; v[u][3] = w.w;
          } else {
            v[u][0] = *reinterpret_cast<const u32*>(a.uc_send + (off - lo));
          }
        } else if (G == 16) {
          mm_ldred4<T, OP>(a.mc_send + off, v[u]);
        } else {
          v[u][0] = mm_ldred1<T, OP>(a.mc_send + off);
        }
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const i64 k = base + (i64)u * nth;
      if (k < n) {
        const i64 off = from + k * G;
        if (COLL == CollReduceScatter) {
          if (G == 16) *reinterpret_cast<uint4*>(a.uc_recv + (off - lo)) = make_uint4(v[u][0], v[u][1], v[u][2], v[u][3]);
          else *reinterpret_cast<u32*>(a.uc_recv + (off - lo)) = v[u][0];
        } else if (G == 16) {
          mm_st4(a.mc_recv + off, v[u]);
        } else {
          mm_st1(a.mc_recv + off, v[u][0]);
        }
      }
    }
  }
}

// This rank's range [lo, hi): 16-byte granules from lo (vec; lo is 16-byte aligned in
// every address space then) and 4-byte granules for the rest.
template <class T, int OP, int COLL>
__device__ __forceinline__ void nvls_run(const NvlsArgs& a) {
  nvls_barrier(a, 0);
  const i64 lo = a.lo_bytes, hi = a.hi_bytes;
  const i64 mid = a.vec ? lo + (hi - lo) / 16 * 16 : lo;
  if (a.vec) nvls_span<T, OP, COLL, 16>(a, lo, mid);
  nvls_span<T, OP, COLL, 4>(a, mid, hi);
  nvls_barrier(a, 1);
}

}  // namespace rdev
