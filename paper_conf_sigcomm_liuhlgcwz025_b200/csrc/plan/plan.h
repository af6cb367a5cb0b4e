// ResCCL planner: global dependency analysis, HPDS primitive-level scheduling,
// task->primitive translation, state-based TB allocation and fusion.
//
//  build_dag   P:L705-737, P:L813-826, P:L1420-1440, P:L1657-1664 (reading R1)
//  hpds        Alg. 1, P:L1579-1629, P:L1680-1774 (readings R2-R4)
//  round_robin P:L2361-2377 (baseline of Fig. 10b)
//  lower       P:L1810-1824 (translation), Eq. 7 (state-based
//              allocation), SURVEY §8(a) a4 (recvReduceSend / recvCopySend fusion)
//
// Every rank computes the identical plan from the identical IR (host only,
// deterministic), as in the paper's offline compiler.
#pragma once

#include <string>
#include <utility>
#include <vector>

#include "ir.h"

namespace resccl {

enum class LinkModel { Pair, Port };

struct Dag {
  std::vector<std::pair<int, int>> edges;      // sorted (u, v)
  std::vector<std::vector<int>> edge_ranks;    // ranks of the inducing locations, per edge
  std::vector<std::vector<int>> preds;         // per task
  std::vector<std::vector<int>> succs;         // per task
};

void validate_ir(const Ir& ir);            // I6; throws PlanError
Dag build_dag(const Ir& ir);               // throws PlanError on same-step conflicts
std::vector<std::vector<int>> hpds(const Ir& ir, const Dag& dag, LinkModel m);
std::vector<std::vector<int>> round_robin(const Ir& ir, const Dag& dag, LinkModel m);

enum Buf : int { BufNone = -1, BufSend = 0, BufRecv = 1, BufScratch = 2 };

// Primitive kinds: the paper's send / recv / recvReduceCopy (rrc) and the fused
// recvReduceSend (rrs), recvReduceCopySend (rrcs), recvCopySend (rcs), recvSend
// (rs, forward without a local store), plus a local copy for outputs no transfer writes.
enum PrimFlags : int {
  kRecv = 1,     // consumes a payload from an incoming FIFO
  kSend = 2,     // produces a payload into an outgoing FIFO
  kReduce = 4,   // value = local (+) incoming
  kStore = 8,    // stores the value locally
  kCopy = 16,    // local copy send buffer -> receive buffer
  // direct transport (reading R23): no FIFO staging.  recv tasks are pushed by the
  // sender straight into the receiver's location once the receiver posted "writable";
  // rrc tasks are pulled: the sender only posts "readable" and the receiver reads the
  // sender's location; the sender's completion is the receiver's read acknowledgement.
  kDirect = 32,
  kPull = 64,      // with kDirect + kRecv: the incoming payload is read from the peer (rrc task)
  kSendPull = 128, // with kDirect + kSend: the outgoing task is pulled -- post "readable" only
};

struct Prim {
  int flags = 0;
  int chunk = 0;
  int pc = -1;          // pipeline index (sub-pipeline number)
  int recv_task = -1;   // task whose payload is consumed
  int send_task = -1;   // task whose payload is produced
  int src_buf = BufNone;  // local operand
  int dst_buf = BufNone;  // local store target
  int cta = 0;
  int lane = 0;         // 0 = send lane, 1 = recv lane
  std::vector<int> deps;  // prim ids on this rank whose same-micro-batch completion is awaited
  std::vector<int> ack_deps;  // direct mode: pull-send prims whose completion is the peer's ack
  int rem_buf = BufNone;  // direct mode: buffer of the peer location a pull reads
  int rem_out = BufNone;  // direct mode: buffer of the peer location a push writes
  bool has_counter = false;
  // lane index (in its lane's list) of the last earlier same-lane primitive a dependency
  // on which was dropped as implied by lane order, or -1 (codegen: writable lookahead, R30)
  int implied_max = -1;
  const char* kind_name() const;
};

struct Conn {
  int peer;
  int dir;  // 0 send, 1 recv
  bool operator==(const Conn& o) const { return peer == o.peer && dir == o.dir; }
  bool operator<(const Conn& o) const { return dir != o.dir ? dir < o.dir : peer < o.peer; }
};

struct RankPlan {
  std::vector<Prim> prims;
  std::vector<std::pair<std::vector<int>, std::vector<int>>> ctas;  // (send lane, recv lane)
  std::vector<std::vector<Conn>> send_groups, recv_groups;
  std::vector<std::pair<Conn, std::vector<int>>> activity;  // connection -> active pipeline indices
  int n_connections = 0;
  int paper_tbs() const { return (int)(send_groups.size() + recv_groups.size()); }
};

struct Plan {
  Ir ir;
  LinkModel model = LinkModel::Pair;
  Dag dag;
  std::vector<std::vector<int>> pr;  // Pr = [Pc0, Pc1, ...]
  std::vector<int> pidx;             // task -> pipeline index
  std::vector<RankPlan> ranks;
  bool fused = false;
  bool direct = false;
  bool pushreduce = false;  // direct plan whose rrc tasks keep the staged FIFO (R31)
  // FIFO order of every link: tasks sorted by pipeline index
  std::vector<int> link_pos;  // task -> position on its link
  std::vector<int> link_len;  // task -> #tasks on its link
};

Plan lower(const Ir& ir, LinkModel m, bool fuse, const std::vector<std::vector<int>>* pr = nullptr,
           bool direct = false, bool pushreduce = false);

// Control-only blocking simulation of the lowered plan (I4).  Returns true if every
// lane completes for FIFO depth K and n_mb micro-batches.
bool deadlock_free(const Plan& p, int K, int n_mb, std::string* why = nullptr);

std::string plan_json(const Plan& p);

}  // namespace resccl
