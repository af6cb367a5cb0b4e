// ResCCL lightweight kernel generation (§4.5).
//
// The three-level paradigm "rank -> TB -> pipeline index" is lowered into one
// CUDA translation unit per schedule: block b -> (rank, TB, instance); each TB's
// send and recv lanes are straight-line lists of `rdev::run<T, OP, Pk>` calls
// sorted by pipeline index, every Pk a constexpr descriptor (chunk, buffers, FIFO
// offsets, link positions, counters, dependency waits).  There is no interpreter:
// every peer, chunk id, FIFO offset and dependency is a compile-time constant;
// only buffers, sizes and the micro-batch base are kernel arguments.
#pragma once

#include <cstdint>
#include <map>
#include <string>
#include <vector>

#include "plan.h"

namespace resccl {

struct Layout {
  int K = 4;               // FIFO depth (slots per link and instance)
  int I = 1;               // instances (paper's nChannels / "Instance")
  int64_t chunk_bytes = 1 << 20;  // Table 2 ChunkSize
  int64_t slot = 0;        // bytes per FIFO slot
  int64_t flagstride = 0;  // bytes of flags per (link, instance)
  // per rank
  std::vector<std::map<int, int>> send_idx, recv_idx;  // peer -> connection index
  std::vector<std::vector<int>> ctr_slot;              // prim -> counter slot (-1: none)
  std::vector<int64_t> cred_base, ctr_base, flag_base, data_base, bytes;
  // Flag rings: one per (receive connection, sending lane).  A link whose sends come
  // from several lanes (fused forwards beside plain sends) gets one ring per lane, so
  // each ring is posted in increasing position order and "flag >= pos + 1" implies that
  // pos was posted (R26).  task_sub[t] = ring of task t within its connection.
  std::vector<std::vector<int>> flag_conn;  // per rank: first ring of each receive connection
  std::vector<int> task_sub;
  int64_t region_bytes = 0;  // max over ranks (regions sit at the same arena offset)
  int64_t done_off = 0;      // exit-barrier counter (direct transport across processes)
  // TB geometry
  std::vector<int> ctas;        // per rank
  std::vector<int> pair_start;  // per rank: index of (rank, cta 0) among all (rank, cta) pairs
  int total_pairs = 0;
};

Layout make_layout(const Plan& p, int K, int I, int64_t chunk_bytes);

struct CodegenOpts {
  int rank_lo = 0, rank_hi = 0;  // ranks [lo, hi) get code
  bool gpu_scope = false;        // all ranks on one device (virtual ranks): .gpu-scope flags
  int nwarps = 16;
  int tma = 1;                   // bulk-copy (TMA) data path for non-reducing primitives
  int tma_tile = 24576;          // bytes per staged tile
  int tma_stages = 2;            // stages per lane (the CTA pool holds 2x)
  int trace = 0;                 // per-lane lifetime / wait timers (TB utilisation, Table 3)
  int phase = 0;                 // per-(primitive, micro-batch) %globaltimer phase records
  int relay_bypass = 1;          // wait on a flags-only push receive's flag, not its counter (R29)
  int lookahead = 1;             // post push receives' "writable" credits ahead of the lane (R30)
  int l2hint = 1;                // L2 evict_last on FIFO writes, evict_first on streams
  int tma_min = 32768;           // slices below this many bytes use the register path
  int backoff = 1;               // nanosleep back-off while polling flags
  int pollacq = 0;               // poll flags with ld.acquire (no separate confirming acquire)
  int jitter = 0;                // debug fault injector: random delays around every sync
  int prefetch = 0;              // micro-batches of local operand prefetched into L2 ahead (off: r01)
  int pool_cap = 0;              // stages of the CTA pool one lane may hold (0 = all)
  int ring = 0;                  // lane-private stage rings instead of the shared CTA pool
  int bulkred = 0;               // in-place reduces: bulk-add the incoming tile in L2
  int cpoll = 0;                 // combine warps: 1 = one polling warp + named barrier
  int early_exit = 1;            // the lane engine leaves its loop right after the last post
  int post_group = 1;            // consecutive dependency-free pull-sends posted as one group
  int split_fence = 1;           // one-sided release / acquire fences
  int store_lag = 1;             // bulk stores a lane lets drain before it blocks to reuse a stage
  int exit_barrier = 0;          // direct transport across processes: a rank's kernel ends only
                                 // after every peer's blocks finished touching its buffers
};

// dynamic shared memory the generated kernel needs (both lanes' TMA staging)
// (a pool of 2 x stages stages of (A tile + B tile), shared by the CTA's two lanes)
inline int codegen_smem_bytes(const CodegenOpts& o) {
  return o.tma ? 4 * o.tma_stages * o.tma_tile : 0;
}

// Device code (without the L0 library text, which the runtime prepends).
std::string codegen(const Plan& p, const Layout& L, const CodegenOpts& o);

// Host geometry of one call (reading R6; identical to the oracle's).
struct Geometry {
  int64_t C = 0, M = 0, Mi = 0;
  int n_mb = 0;
};
Geometry geometry(Coll coll, int nranks, int64_t count, int elt, int64_t chunk_bytes, int instances);

}  // namespace resccl
