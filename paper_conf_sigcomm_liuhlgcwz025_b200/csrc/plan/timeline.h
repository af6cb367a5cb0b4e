// Wall-clock timeline of a lowered plan under the paper's alpha-beta cost model with
// link contention (Eq. 1) and task-level execution (Eq. 5),
// and the state-based TB merge evaluated on wall-clock activity (Eq. 7's
// active_l(t)).  Host only; the f2 row of SURVEY §8.
//
// Model (reading R27):
//  * every lane (CTA lane x instance) runs its primitive list in order; invocation j of
//    a primitive starts once the blocking-model conditions of the plan check hold
//    (local dependency counters, payload / FIFO credit, direct-mode writable/readable
//    flags) and ends after its work is done; its effects (payload posted, credit
//    returned, counter bumped) apply at the end;
//  * work = alpha + c * beta when the invocation moves c bytes over a link (a staged or
//    pushed send, a pulled receive), alpha otherwise (a FIFO drain, a flag post, a
//    local copy); a push receiver's "writable" post is instantaneous;
//  * link contention (Eq. 1): z invocations moving data on one link (pair model: the
//    (src, dst) connection; port model: the sender's egress and the receiver's
//    ingress port) share it, each progressing at rate 1/z; an invocation that starts
//    on a link already carrying others first pays gamma * L(z) / n_mb with
//    L(z) = z - 1, so a task of n_mb invocations pays Eq. 1's L(z) * gamma once;
//  * lane activity intervals give active_l(t) for each connection; connections of one
//    direction whose activity never overlaps are merged greedily (first start
//    first), which is Eq. 7 on the wall clock rather than on pipeline indices.
#pragma once

#include <string>
#include <vector>

#include "plan.h"

namespace resccl {

struct TimelineParams {
  double alpha = 2e-6;        // s: start-up overhead of one invocation
  double beta = 1.0 / 900e9;  // s/byte: inverse link bandwidth
  double gamma = 2e-6;        // s: contention constant of Eq. 1
  double c = 1 << 20;         // bytes moved per invocation (micro-batch slice of one instance)
  int n_mb = 1;               // micro-batches
  int K = 4;                  // FIFO depth (staged transport)
  int instances = 1;          // instance copies sharing the links
};

struct TimelineResult {
  double makespan = 0;                                  // s
  std::vector<double> lane_busy;                        // s, per traced lane (instance 0 first)
  std::vector<std::vector<std::vector<std::pair<double, double>>>> conn_active;  // rank -> conn -> intervals
  std::vector<std::vector<std::pair<int, int>>> conns;  // rank -> (peer, dir 0 send / 1 recv)
  std::vector<int> merged_send, merged_recv;            // rank -> lanes after the wall-clock merge
  double max_z = 1;                                     // largest contention seen
};

TimelineResult simulate_timeline(const Plan& p, const TimelineParams& tp);
std::string timeline_json(const Plan& p, const TimelineParams& tp, const TimelineResult& r);

}  // namespace resccl
