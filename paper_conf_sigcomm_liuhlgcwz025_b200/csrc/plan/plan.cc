// ResCCL planner implementation.  See plan.h for the passages each step follows.
#include "plan.h"

#include <algorithm>
#include <deque>
#include <map>
#include <set>
#include <sstream>
#include <tuple>

namespace resccl {

const char* Prim::kind_name() const {
  if (flags & kCopy) return "copy";
  if (flags & kDirect) {
    if (!(flags & kRecv)) return (flags & kSendPull) ? "psend" : "dsend";
    if (!(flags & kSend)) return (flags & kPull) ? "prrc" : "drecv";
    if (flags & kPull) return (flags & kSendPull) ? "prrc_p" : "prrc_d";
    return (flags & kSendPull) ? "drecv_p" : "drecv_d";
  }
  bool rv = flags & kRecv, sd = flags & kSend, red = flags & kReduce, st = flags & kStore;
  if (!rv) return "send";
  if (!sd) return red ? "rrc" : "recv";
  if (red) return st ? "rrcs" : "rrs";
  return st ? "rcs" : "rs";
}

// ----------------------------------------------------------------------------- IR checks
void validate_ir(const Ir& ir) {
  if (ir.nranks < 1) throw PlanError("nranks must be >= 1");
  if (ir.nchunks != ir.nranks) throw PlanError("nchunks must equal nranks (R19)");
  if (ir.nwarps < 2 || ir.nwarps > 32 || ir.nwarps % 2) throw PlanError("nwarps must be even, 2..32");
  std::set<std::tuple<int, int, int, int, int>> seen;
  for (auto& x : ir.t) {
    if (x.src < 0 || x.src >= ir.nranks || x.dst < 0 || x.dst >= ir.nranks)
      throw PlanError("transfer rank out of range");
    if (x.chunk < 0 || x.chunk >= ir.nchunks) throw PlanError("transfer chunk out of range");
    if (x.src == x.dst) throw PlanError("self transfer");
    if (x.step < 0) throw PlanError("negative step");
    if (ir.coll == Coll::AllGather && x.op == Op::Rrc) throw PlanError("allgather algorithms use recv only");
    if (!seen.insert({x.src, x.dst, x.step, x.chunk, (int)x.op}).second) throw PlanError("duplicate transfer");
  }
  if (ir.coll == Coll::AllGather) {  // write-once, no undefined reads
    std::map<std::pair<int, int>, int> first_w;
    for (auto& x : ir.t) {
      if (x.dst == x.chunk) throw PlanError("allgather overwrites the owner's chunk");
      if (!first_w.emplace(std::make_pair(x.dst, x.chunk), x.step).second)
        throw PlanError("allgather location written twice");
    }
    for (auto& x : ir.t) {
      if (x.src == x.chunk) continue;
      auto it = first_w.find({x.src, x.chunk});
      if (it == first_w.end() || it->second >= x.step) throw PlanError("read of an undefined location");
    }
  }
}

// ----------------------------------------------------------------------------- DAG (R1)
Dag build_dag(const Ir& ir) {
  validate_ir(ir);
  const int T = (int)ir.t.size();
  // location -> (step, task, kind) with kind 0 = R, 1 = W, 2 = RW
  std::map<std::pair<int, int>, std::vector<std::tuple<int, int, int>>> by_loc;
  for (int i = 0; i < T; ++i) {
    auto& x = ir.t[i];
    by_loc[{x.src, x.chunk}].push_back({x.step, i, 0});
    by_loc[{x.dst, x.chunk}].push_back({x.step, i, x.op == Op::Rrc ? 2 : 1});
  }
  std::map<std::pair<int, int>, std::set<int>> er;
  for (auto& kv : by_loc) {
    auto acc = kv.second;
    std::sort(acc.begin(), acc.end());
    int last_w = -1;
    std::vector<int> readers;
    size_t a = 0;
    while (a < acc.size()) {
      size_t b = a;
      bool has_w = false;
      while (b < acc.size() && std::get<0>(acc[b]) == std::get<0>(acc[a])) {
        has_w |= std::get<2>(acc[b]) != 0;
        ++b;
      }
      if (has_w && b - a > 1)
        throw PlanError("same-step conflict at location <" + std::to_string(kv.first.first) + "," +
                        std::to_string(kv.first.second) + "> step " + std::to_string(std::get<0>(acc[a])));
      if (!has_w) {
        for (size_t k = a; k < b; ++k) {
          int i = std::get<1>(acc[k]);
          if (last_w >= 0) er[{last_w, i}].insert(kv.first.first);
          readers.push_back(i);
        }
      } else {
        int i = std::get<1>(acc[a]);
        if (last_w >= 0) er[{last_w, i}].insert(kv.first.first);
        for (int rd : readers)
          if (rd != i) er[{rd, i}].insert(kv.first.first);
        last_w = i;
        readers.clear();
      }
      a = b;
    }
  }
  Dag d;
  d.preds.assign(T, {});
  d.succs.assign(T, {});
  for (auto& kv : er) {
    d.edges.push_back(kv.first);
    d.edge_ranks.emplace_back(kv.second.begin(), kv.second.end());
    d.preds[kv.first.second].push_back(kv.first.first);
    d.succs[kv.first.first].push_back(kv.first.second);
  }
  return d;
}

// ----------------------------------------------------------------------------- HPDS (Alg. 1)
using LinkKey = std::pair<int, int>;
static void task_links(const Transfer& x, LinkModel m, int n, LinkKey out[2], int* cnt) {
  if (m == LinkModel::Pair) {
    out[0] = {0, x.src * n + x.dst};
    *cnt = 1;
  } else {
    out[0] = {1, x.src};
    out[1] = {2, x.dst};
    *cnt = 2;
  }
}

// Incremental list scheduler: per-chunk ready sets ordered by (step, src, dst) and a
// remaining-predecessor count per task, so a task becomes ready right after its last
// predecessor leaves G (R4: before the next inner iteration).  Alg. 1's chunk choice
// (line 9) uses an ordered set of (priority, ChunkId).  O(T log T + #Pc * C log C).
static std::vector<std::vector<int>> list_schedule(const Ir& ir, const Dag& dag, LinkModel m, bool rr) {
  const int T = (int)ir.t.size(), N = ir.nranks;
  auto cmp = [&](int a, int b) {
    auto& x = ir.t[a];
    auto& y = ir.t[b];
    return std::tie(x.step, x.src, x.dst, a) < std::tie(y.step, y.src, y.dst, b);
  };
  std::map<int, std::set<int, decltype(cmp)>> ready;
  std::vector<int> npred(T);
  std::set<int> chunkset;
  for (auto& x : ir.t) chunkset.insert(x.chunk);
  std::vector<int> chunks(chunkset.begin(), chunkset.end());
  for (int c : chunks) ready.emplace(c, std::set<int, decltype(cmp)>(cmp));
  for (int i = 0; i < T; ++i) {
    npred[i] = (int)dag.preds[i].size();
    if (npred[i] == 0) ready.at(ir.t[i].chunk).insert(i);
  }
  std::map<int, int> prio;
  for (int c : chunks) prio[c] = 0;
  int left = T;
  std::vector<std::vector<int>> Pr;
  while (left > 0) {                                   // line 5
    std::vector<int> pc;                               // line 6
    std::set<LinkKey> used;
    auto take = [&](int C) {                           // lines 10-15: NodeList of chunk C
      std::vector<int> nl;
      for (int i : ready.at(C)) {
        LinkKey lk[2];
        int nk;
        task_links(ir.t[i], m, N, lk, &nk);
        bool free = true;
        for (int k = 0; k < nk; ++k)
          if (used.count(lk[k])) free = false;
        if (free) {
          nl.push_back(i);
          for (int k = 0; k < nk; ++k) used.insert(lk[k]);
        }
      }
      return nl;
    };
    auto remove = [&](const std::vector<int>& nl) {    // line 22: G.remove(NodeList)
      for (int i : nl) {
        ready.at(ir.t[i].chunk).erase(i);
        --left;
        for (int s : dag.succs[i])
          if (--npred[s] == 0) ready.at(ir.t[s].chunk).insert(s);
      }
    };
    if (!rr) {
      // line 7: F = all true; line 9: highest priority, ties -> lowest ChunkId
      std::set<std::pair<int, int>> Q;                 // (-priority, chunk) of flagged chunks
      for (int c : chunks) Q.insert({-prio[c], c});
      while (!Q.empty()) {                             // line 8
        int C = Q.begin()->second;
        auto nl = take(C);
        if (nl.empty()) {
          Q.erase(Q.begin());                          // line 17
        } else {
          pc.insert(pc.end(), nl.begin(), nl.end());   // line 19
          Q.erase(Q.begin());
          prio[C] -= 1;                                // lines 20-21
          Q.insert({-prio[C], C});
          remove(nl);
        }
      }
    } else {                                           // RR baseline: fixed ascending order
      bool progress = true;
      while (progress) {
        progress = false;
        for (int C : chunks) {
          auto nl = take(C);
          if (!nl.empty()) {
            pc.insert(pc.end(), nl.begin(), nl.end());
            remove(nl);
            progress = true;
          }
        }
      }
    }
    if (pc.empty()) throw PlanError("scheduler made no progress (cyclic dependencies)");
    Pr.push_back(pc);                                  // line 25
  }
  return Pr;
}

std::vector<std::vector<int>> hpds(const Ir& ir, const Dag& dag, LinkModel m) {
  return list_schedule(ir, dag, m, false);
}
std::vector<std::vector<int>> round_robin(const Ir& ir, const Dag& dag, LinkModel m) {
  return list_schedule(ir, dag, m, true);
}

// ----------------------------------------------------------------------------- lowering
static bool is_output(Coll c, int r, int chunk) { return c != Coll::ReduceScatter || chunk == r; }
static int write_buf(Coll c, int r, int chunk) {
  return (c == Coll::ReduceScatter && chunk != r) ? BufScratch : BufRecv;
}

// Greedy merge of connections with disjoint activity (Eq. 7), ordered by (first
// active pipeline index, peer).
static std::vector<std::vector<Conn>> greedy_merge(std::vector<std::pair<Conn, std::set<int>>> conns) {
  std::sort(conns.begin(), conns.end(), [](auto& a, auto& b) {
    int fa = *a.second.begin(), fb = *b.second.begin();
    return std::tie(fa, a.first.peer) < std::tie(fb, b.first.peer);
  });
  std::vector<std::vector<Conn>> groups;
  std::vector<std::set<int>> gact;
  for (auto& cn : conns) {
    bool placed = false;
    for (size_t g = 0; g < groups.size() && !placed; ++g) {
      bool disjoint = true;
      for (int k : cn.second)
        if (gact[g].count(k)) { disjoint = false; break; }
      if (disjoint) {
        groups[g].push_back(cn.first);
        gact[g].insert(cn.second.begin(), cn.second.end());
        placed = true;
      }
    }
    if (!placed) {
      groups.push_back({cn.first});
      gact.push_back(cn.second);
    }
  }
  return groups;
}

namespace {
struct Raw {  // unfused translation of one rank
  std::vector<Prim> prims;
  std::vector<std::set<int>> deps;  // DAG-derived local deps (raw prim ids)
};
}  // namespace

static void build_ranks(Plan& P, const std::vector<Raw>& raw, const std::vector<std::map<int, int>>& absorbed,
                        const std::map<std::pair<int, int>, std::vector<std::tuple<int, int, int>>>& loc_acc,
                        const std::set<std::pair<int, int>>& written) {
  const Ir& ir = P.ir;
  const int N = ir.nranks;
  for (int r = 0; r < N; ++r) {
    RankPlan& RP = P.ranks[r];
    std::vector<Prim> ps = raw[r].prims;
    const auto& fused_into = absorbed[r];  // send raw id -> recv raw id
    std::map<int, int> fused_rev;          // recv raw id -> send raw id
    for (auto& kv : fused_into) fused_rev[kv.second] = kv.first;
    for (auto& kv : fused_into) {
      Prim& a = ps[kv.second];
      const Prim& b = ps[kv.first];
      int t1 = a.recv_task, t2 = b.send_task;
      const auto& acc = loc_acc.at({r, a.chunk});
      size_t pos = 0;
      while (!(std::get<1>(acc[pos]) == t1 && std::get<2>(acc[pos]) != 0)) ++pos;
      std::set<int> readers;
      bool final_ = true;
      for (size_t k = pos + 1; k < acc.size(); ++k) {
        int i = std::get<1>(acc[k]), kind = std::get<2>(acc[k]);
        if (kind == 0) {
          readers.insert(i);
        } else {
          if (kind == 2) readers.insert(i);
          final_ = false;
          break;
        }
      }
      bool store = (final_ && is_output(ir.coll, r, a.chunk)) || readers != std::set<int>{t2};
      a.send_task = t2;
      a.flags |= kSend;
      if (a.flags & kDirect) {
        // direct: the next hop pulls from / is pushed from our location, so the value
        // stays stored; the send part keeps its push / pull mode
        a.flags |= (b.flags & kSendPull);
        a.rem_out = b.rem_out;
        if (!(a.flags & kPull)) a.src_buf = a.dst_buf;  // push receiver forwards its location
      } else if (!store) {
        a.flags &= ~kStore;
        a.dst_buf = BufNone;
      }
    }
    // final prim list: copies first, then all non-absorbed prims in raw order.  An output
    // location never written on r (AllGather's own chunk) is copied by the first
    // data-moving send of it from the send buffer -- it stores its tile locally too (one
    // read, overlapped with the ring) -- else by a separate copy primitive.  Nothing reads
    // that location from the receive buffer during the collective, so when the copy
    // lands does not matter.
    std::vector<Prim> fin;
    std::vector<int> raw_of;  // final index -> raw id (-1 for copies)
    for (int c = 0; c < ir.nchunks; ++c)
      if (is_output(ir.coll, r, c) && !written.count({r, c})) {
        bool folded = false;
        for (int i = 0; i < (int)ps.size() && !folded; ++i) {
          Prim& q = ps[i];
          if (fused_into.count(i) || q.chunk != c || !(q.flags & kSend) || (q.flags & kRecv) ||
              (q.flags & kSendPull) || q.src_buf != BufSend)
            continue;
          q.flags |= kStore;
          q.dst_buf = BufRecv;
          folded = true;
        }
        if (folded) continue;
        Prim cp;
        cp.flags = kCopy;
        cp.chunk = c;
        cp.pc = -1;
        cp.src_buf = BufSend;
        cp.dst_buf = BufRecv;
        cp.cta = 0;
        cp.lane = 1;
        fin.push_back(cp);
        raw_of.push_back(-1);
      }
    std::map<int, int> newid;
    for (int i = 0; i < (int)ps.size(); ++i) {
      if (fused_into.count(i)) continue;
      newid[i] = (int)fin.size();
      fin.push_back(ps[i]);
      raw_of.push_back(i);
    }
    auto remap = [&](int raw_id) {
      auto it = fused_into.find(raw_id);
      return newid.at(it == fused_into.end() ? raw_id : it->second);
    };
    // direct mode: a dependency on a pull-send (also when absorbed into a fused prim)
    // completes with the receiver's ack of that send's link -> ack dependency
    auto is_ack = [&](int raw_id) {
      return P.direct && (ps[raw_id].flags & kSendPull) && !(ps[raw_id].flags & kRecv);
    };
    for (int k = 0; k < (int)fin.size(); ++k) {
      int old = raw_of[k];
      if (old < 0) continue;
      std::set<int> ds, as;
      auto add = [&](int d) { (is_ack(d) ? as : ds).insert(remap(d)); };
      for (int d : raw[r].deps[old]) add(d);
      auto fr = fused_rev.find(old);
      if (fr != fused_rev.end())
        for (int d : raw[r].deps[fr->second]) add(d);
      ds.erase(k);
      as.erase(k);
      fin[k].deps.assign(ds.begin(), ds.end());
      fin[k].ack_deps.assign(as.begin(), as.end());
    }
    int ncta = std::max<int>({(int)RP.send_groups.size(), (int)RP.recv_groups.size(), 1});
    RP.ctas.assign(ncta, {});
    for (int lane = 0; lane < 2; ++lane)
      for (int c = 0; c < ncta; ++c) {
        std::vector<int> l;
        for (int k = 0; k < (int)fin.size(); ++k)
          if (fin[k].lane == lane && fin[k].cta == c) l.push_back(k);
        std::stable_sort(l.begin(), l.end(), [&](int a, int b) { return fin[a].pc < fin[b].pc; });
        (lane == 0 ? RP.ctas[c].first : RP.ctas[c].second) = l;
      }
    // (ack dependencies are never implied by lane order: a pull-send returns before the read)
    // drop dependencies implied by lane order
    std::map<int, std::tuple<int, int, int>> where;
    for (int c = 0; c < ncta; ++c) {
      for (int k = 0; k < (int)RP.ctas[c].first.size(); ++k) where[RP.ctas[c].first[k]] = {c, 0, k};
      for (int k = 0; k < (int)RP.ctas[c].second.size(); ++k) where[RP.ctas[c].second[k]] = {c, 1, k};
    }
    for (int k = 0; k < (int)fin.size(); ++k) {
      auto me = where[k];
      std::vector<int> keep;
      for (int d : fin[k].deps) {
        auto w = where[d];
        bool implied = std::get<0>(w) == std::get<0>(me) && std::get<1>(w) == std::get<1>(me) &&
                       std::get<2>(w) < std::get<2>(me);
        if (!implied) keep.push_back(d);
        else fin[k].implied_max = std::max(fin[k].implied_max, std::get<2>(w));
      }
      fin[k].deps = keep;
    }
    for (auto& p : fin)
      for (int d : p.deps) fin[d].has_counter = true;
    RP.prims = std::move(fin);
  }
}

Plan lower(const Ir& ir, LinkModel m, bool fuse, const std::vector<std::vector<int>>* pr_in, bool direct,
           bool pushreduce) {
  Plan P;
  P.ir = ir;
  P.model = m;
  P.direct = direct;
  P.pushreduce = direct && pushreduce;
  P.dag = build_dag(ir);
  P.pr = pr_in ? *pr_in : hpds(ir, P.dag, m);
  const int T = (int)ir.t.size(), N = ir.nranks;
  P.pidx.assign(T, -1);
  for (int k = 0; k < (int)P.pr.size(); ++k)
    for (int i : P.pr[k]) P.pidx[i] = k;
  for (int i = 0; i < T; ++i)
    if (P.pidx[i] < 0) throw PlanError("task missing from the pipeline");
  // link FIFO order
  {
    std::map<std::pair<int, int>, std::vector<int>> links;
    for (int i = 0; i < T; ++i) links[{ir.t[i].src, ir.t[i].dst}].push_back(i);
    P.link_pos.assign(T, 0);
    P.link_len.assign(T, 0);
    for (auto& kv : links) {
      auto v = kv.second;
      std::stable_sort(v.begin(), v.end(), [&](int a, int b) { return P.pidx[a] < P.pidx[b]; });
      for (int k = 0; k < (int)v.size(); ++k) {
        P.link_pos[v[k]] = k;
        P.link_len[v[k]] = (int)v.size();
      }
    }
  }
  // location accesses and first writes (send-buffer vs receive-buffer reads, R18)
  std::map<std::pair<int, int>, std::vector<std::tuple<int, int, int>>> loc_acc;
  std::map<std::pair<int, int>, int> first_w;
  std::set<std::pair<int, int>> written;
  for (int i = 0; i < T; ++i) {
    auto& x = ir.t[i];
    loc_acc[{x.src, x.chunk}].push_back({x.step, i, 0});
    loc_acc[{x.dst, x.chunk}].push_back({x.step, i, x.op == Op::Rrc ? 2 : 1});
    auto it = first_w.find({x.dst, x.chunk});
    if (it == first_w.end() || x.step < it->second) first_w[{x.dst, x.chunk}] = x.step;
    written.insert({x.dst, x.chunk});
  }
  for (auto& kv : loc_acc) std::sort(kv.second.begin(), kv.second.end());
  auto read_buf = [&](int r, int c, int step) {
    auto it = first_w.find({r, c});
    if (it != first_w.end() && it->second < step) return write_buf(ir.coll, r, c);
    return (int)BufSend;
  };
  // translation
  std::vector<Raw> raw(N);
  std::vector<std::pair<int, int>> send_of(T), recv_of(T);
  for (int i = 0; i < T; ++i) {
    auto& x = ir.t[i];
    Prim s;
    s.flags = kSend;
    s.chunk = x.chunk;
    s.pc = P.pidx[i];
    s.send_task = i;
    s.src_buf = read_buf(x.src, x.chunk, x.step);
    send_of[i] = {x.src, (int)raw[x.src].prims.size()};
    raw[x.src].prims.push_back(s);
    Prim rv;
    rv.flags = kRecv | kStore | (x.op == Op::Rrc ? kReduce : 0);
    rv.chunk = x.chunk;
    rv.pc = P.pidx[i];
    rv.recv_task = i;
    rv.dst_buf = write_buf(ir.coll, x.dst, x.chunk);
    rv.src_buf = x.op == Op::Rrc ? read_buf(x.dst, x.chunk, x.step) : BufNone;
    rv.lane = 1;
    if (direct && !(x.op == Op::Rrc && pushreduce)) {  // (push-reduce, R31: rrc tasks stay staged)
      if (x.op == Op::Rrc) {  // pull: receiver reads the sender's location
        s.flags |= kDirect | kSendPull;
        rv.flags |= kDirect | kPull;
        rv.rem_buf = s.src_buf;
      } else {                // push: sender writes the receiver's location
        s.flags |= kDirect;
        s.rem_out = rv.dst_buf;
        rv.flags = kRecv | kDirect;
      }
      raw[x.src].prims[send_of[i].second] = s;
    }
    recv_of[i] = {x.dst, (int)raw[x.dst].prims.size()};
    raw[x.dst].prims.push_back(rv);
  }
  for (int r = 0; r < N; ++r) raw[r].deps.assign(raw[r].prims.size(), {});
  // state-based TB allocation (Eq. 7)
  P.ranks.assign(N, {});
  std::vector<std::map<Conn, std::set<int>>> act(N);
  for (int i = 0; i < T; ++i) {
    act[ir.t[i].src][{ir.t[i].dst, 0}].insert(P.pidx[i]);
    act[ir.t[i].dst][{ir.t[i].src, 1}].insert(P.pidx[i]);
  }
  std::vector<std::map<Conn, int>> lane_of(N);
  for (int r = 0; r < N; ++r) {
    std::vector<std::pair<Conn, std::set<int>>> sa, ra;
    for (auto& kv : act[r]) (kv.first.dir == 0 ? sa : ra).push_back(kv);
    auto& RP = P.ranks[r];
    RP.send_groups = greedy_merge(sa);
    RP.recv_groups = greedy_merge(ra);
    RP.n_connections = (int)act[r].size();
    for (auto& kv : act[r]) RP.activity.push_back({kv.first, std::vector<int>(kv.second.begin(), kv.second.end())});
    for (int g = 0; g < (int)RP.send_groups.size(); ++g)
      for (auto& c : RP.send_groups[g]) lane_of[r][c] = g;
    for (int g = 0; g < (int)RP.recv_groups.size(); ++g)
      for (auto& c : RP.recv_groups[g]) lane_of[r][c] = g;
  }
  for (int i = 0; i < T; ++i) {
    auto& x = ir.t[i];
    raw[x.src].prims[send_of[i].second].cta = lane_of[x.src][{x.dst, 0}];
    raw[x.dst].prims[recv_of[i].second].cta = lane_of[x.dst][{x.src, 1}];
  }
  // local dependencies
  auto prim_at = [&](int i, int x) { return ir.t[i].src == x ? send_of[i].second : recv_of[i].second; };
  for (size_t e = 0; e < P.dag.edges.size(); ++e) {
    int u = P.dag.edges[e].first, v = P.dag.edges[e].second;
    for (int x : P.dag.edge_ranks[e]) raw[x].deps[prim_at(v, x)].insert(prim_at(u, x));
  }
  // fusion candidates
  std::vector<std::map<int, int>> absorbed(N), none(N);
  if (fuse) {
    for (int r = 0; r < N; ++r) {
      auto& ps = raw[r].prims;
      std::vector<int> rl;
      for (int k = 0; k < (int)ps.size(); ++k)
        if (ps[k].lane == 1) rl.push_back(k);
      std::stable_sort(rl.begin(), rl.end(), [&](int a, int b) {
        return std::tie(ps[a].cta, ps[a].pc) < std::tie(ps[b].cta, ps[b].pc);
      });
      std::set<int> taken;
      for (int a : rl) {
        int best = -1;
        for (int b = 0; b < (int)ps.size(); ++b) {
          if (ps[b].lane != 0 || ps[b].cta != ps[a].cta || taken.count(b)) continue;
          if ((ps[b].flags & kDirect) != (ps[a].flags & kDirect)) continue;  // only same-mode pairs fuse
          if (raw[r].deps[b] != std::set<int>{a}) continue;
          if (best < 0 || std::make_pair(ps[b].pc, ir.t[ps[b].send_task].dst) <
                              std::make_pair(ps[best].pc, ir.t[ps[best].send_task].dst))
            best = b;
        }
        if (best >= 0) {
          taken.insert(best);
          absorbed[r][best] = a;
        }
      }
    }
  }
  bool any = false;
  for (auto& a : absorbed) any |= !a.empty();
  build_ranks(P, raw, any ? absorbed : none, loc_acc, written);
  P.fused = any;
  if (any) {
    auto check = [&]() {
      bool ok = true;
      for (int nmb : {1, 2, 3, 16}) ok = ok && deadlock_free(P, 1, nmb);
      return ok;
    };
    auto rebuild = [&](const std::vector<std::map<int, int>>& ab) {
      for (auto& RP : P.ranks) {
        RP.prims.clear();
        RP.ctas.clear();
      }
      build_ranks(P, raw, ab, loc_acc, written);
    };
    if (!check()) {
      // direct mode: fusions whose send part only posts "readable" add no wait edge and
      // are kept; push-forwarding fusions can form rendezvous cycles (R21/R23)
      std::vector<std::map<int, int>> safe(N);
      bool any_safe = false;
      if (direct)
        for (int r = 0; r < N; ++r)
          for (auto& kv : absorbed[r])
            if (raw[r].prims[kv.first].flags & kSendPull) {
              safe[r][kv.first] = kv.second;
              any_safe = true;
            }
      if (any_safe) {
        rebuild(safe);
        if (!check()) {
          rebuild(none);
          any_safe = false;
        }
      } else {
        rebuild(none);
      }
      P.fused = any_safe;
    }
  }
  return P;
}

// ----------------------------------------------------------------------------- I4 simulation
// Blocking semantics per (primitive, micro-batch) of a lane; per link a set of posted
// payload positions ("flags") and a monotone credit counter.  Staged: the receiver's
// consumption is the credit; a sender may run K positions ahead.  Direct (R23): a push
// receiver first posts "writable" (credit) once its dependencies hold, then waits for the
// payload; a push sender waits for that credit; a pull sender only posts "readable" and
// its completion (for dependents) is the receiver's read credit.
bool deadlock_free(const Plan& P, int K, int n_mb, std::string* why) {
  const Ir& ir = P.ir;
  struct Proc {
    int r, cta, lane;
    const std::vector<int>* prog;
    int k = 0, j = 0, phase = 0;
  };
  std::vector<Proc> procs;
  for (int r = 0; r < ir.nranks; ++r)
    for (int c = 0; c < (int)P.ranks[r].ctas.size(); ++c) {
      const auto& sl = P.ranks[r].ctas[c].first;
      const auto& rl = P.ranks[r].ctas[c].second;
      if (!sl.empty()) procs.push_back({r, c, 0, &sl});
      if (!rl.empty()) procs.push_back({r, c, 1, &rl});
    }
  std::map<std::pair<int, int>, int> done;  // (rank, prim) -> #micro-batches finished
  std::map<std::pair<int, int>, std::set<long>> produced;
  std::map<std::pair<int, int>, long> credit;
  auto link = [&](int t) { return std::make_pair(ir.t[t].src, ir.t[t].dst); };
  auto pos_of = [&](int t, int j) { return (long)P.link_pos[t] * n_mb + j; };
  auto deps_ok = [&](const Proc& p, const Prim& pm) {
    for (int d : pm.deps)
      if (done[{p.r, d}] < p.j + 1) return false;
    for (int d : pm.ack_deps) {
      int t = P.ranks[p.r].prims[d].send_task;
      if (credit[link(t)] < pos_of(t, p.j) + 1) return false;
    }
    return true;
  };
  auto send_ok = [&](const Proc& p, const Prim& pm) {
    if (!(pm.flags & kSend)) return true;
    long pos = pos_of(pm.send_task, p.j);
    if (!(pm.flags & kDirect)) return pos < credit[link(pm.send_task)] + K;
    if (pm.flags & kSendPull) return true;                      // pull-send: post "readable"
    return credit[link(pm.send_task)] >= pos + 1;               // push: receiver location writable
  };
  auto enabled = [&](Proc& p) {
    if (p.k >= (int)p.prog->size()) return false;
    const Prim& pm = P.ranks[p.r].prims[(*p.prog)[p.k]];
    if (pm.flags & kCopy) return true;
    const bool direct = pm.flags & kDirect, pull = pm.flags & kPull;
    const bool push_recv = direct && (pm.flags & kRecv) && !pull;
    if (push_recv && p.phase == 1)  // push receiver waiting for the payload (and its own send credit)
      return produced[link(pm.recv_task)].count(pos_of(pm.recv_task, p.j)) > 0 && send_ok(p, pm);
    if (!deps_ok(p, pm)) return false;
    if (push_recv) return true;     // phase 0: post "writable"
    if (pm.flags & kRecv)
      if (!produced[link(pm.recv_task)].count(pos_of(pm.recv_task, p.j))) return false;
    return send_ok(p, pm);
  };
  auto fire = [&](Proc& p) {
    int pid = (*p.prog)[p.k];
    const Prim& pm = P.ranks[p.r].prims[pid];
    const bool direct = pm.flags & kDirect, pull = pm.flags & kPull;
    if (direct && (pm.flags & kRecv) && !pull && p.phase == 0) {  // post "writable", keep the micro-batch
      credit[link(pm.recv_task)] = std::max(credit[link(pm.recv_task)], pos_of(pm.recv_task, p.j) + 1);
      p.phase = 1;
      return;
    }
    p.phase = 0;
    if (pm.recv_task >= 0) {
      long pos = pos_of(pm.recv_task, p.j);
      produced[link(pm.recv_task)].erase(pos);
      if (!direct)
        credit[link(pm.recv_task)] += 1;
      else if (pull)
        credit[link(pm.recv_task)] = std::max(credit[link(pm.recv_task)], pos + 1);
    }
    if (pm.send_task >= 0) produced[link(pm.send_task)].insert(pos_of(pm.send_task, p.j));
    if (!(pm.flags & kCopy)) done[{p.r, pid}] = p.j + 1;
    p.j++;
    if (p.j >= ((pm.flags & kCopy) ? 1 : n_mb)) {
      p.k++;
      p.j = 0;
    }
  };
  size_t idx = 0, idle = 0, n = procs.size();
  auto finished = [&]() {
    for (auto& p : procs)
      if (p.k < (int)p.prog->size()) return false;
    return true;
  };
  while (!finished()) {
    Proc& p = procs[idx];
    if (enabled(p)) {
      fire(p);
      idle = 0;
    } else if (++idle > n) {
      if (why) {
        std::ostringstream os;
        os << "deadlock:";
        for (auto& q : procs)
          if (q.k < (int)q.prog->size())
            os << " rank" << q.r << "/cta" << q.cta << (q.lane ? "R" : "S") << "@"
               << P.ranks[q.r].prims[(*q.prog)[q.k]].kind_name() << "#mb" << q.j;
        *why = os.str();
      }
      return false;
    }
    idx = (idx + 1) % n;
  }
  return true;
}

// ----------------------------------------------------------------------------- JSON
static const char* buf_name(int b) {
  switch (b) {
    case BufSend: return "send";
    case BufRecv: return "recv";
    case BufScratch: return "scratch";
  }
  return "none";
}

std::string plan_json(const Plan& P) {
  std::ostringstream o;
  const Ir& ir = P.ir;
  o << "{\"name\":\"" << ir.name << "\",\"coll\":\"" << coll_name(ir.coll) << "\",\"nranks\":" << ir.nranks
    << ",\"model\":\"" << (P.model == LinkModel::Pair ? "pair" : "port") << "\",\"fused\":"
    << (P.fused ? "true" : "false") << ",\"direct\":" << (P.direct ? "true" : "false")
    << ",\"pushreduce\":" << (P.pushreduce ? "true" : "false") << ",\"n_edges\":" << P.dag.edges.size() << ",\"tasks\":[";
  for (size_t i = 0; i < ir.t.size(); ++i) {
    auto& x = ir.t[i];
    o << (i ? "," : "") << "[" << x.src << "," << x.dst << "," << x.step << "," << x.chunk << ",\""
      << (x.op == Op::Rrc ? "rrc" : "recv") << "\"]";
  }
  o << "],\"Pr\":[";
  for (size_t k = 0; k < P.pr.size(); ++k) {
    o << (k ? "," : "") << "[";
    for (size_t i = 0; i < P.pr[k].size(); ++i) o << (i ? "," : "") << P.pr[k][i];
    o << "]";
  }
  o << "],\"ranks\":[";
  for (int r = 0; r < ir.nranks; ++r) {
    const RankPlan& RP = P.ranks[r];
    o << (r ? "," : "") << "{\"n_connections\":" << RP.n_connections << ",\"paper_tbs\":" << RP.paper_tbs()
      << ",\"send_groups\":[";
    for (size_t g = 0; g < RP.send_groups.size(); ++g) {
      o << (g ? "," : "") << "[";
      for (size_t c = 0; c < RP.send_groups[g].size(); ++c) o << (c ? "," : "") << RP.send_groups[g][c].peer;
      o << "]";
    }
    o << "],\"recv_groups\":[";
    for (size_t g = 0; g < RP.recv_groups.size(); ++g) {
      o << (g ? "," : "") << "[";
      for (size_t c = 0; c < RP.recv_groups[g].size(); ++c) o << (c ? "," : "") << RP.recv_groups[g][c].peer;
      o << "]";
    }
    o << "],\"ctas\":[";
    for (size_t c = 0; c < RP.ctas.size(); ++c) {
      o << (c ? "," : "") << "{\"send\":[";
      for (size_t k = 0; k < RP.ctas[c].first.size(); ++k) o << (k ? "," : "") << RP.ctas[c].first[k];
      o << "],\"recv\":[";
      for (size_t k = 0; k < RP.ctas[c].second.size(); ++k) o << (k ? "," : "") << RP.ctas[c].second[k];
      o << "]}";
    }
    o << "],\"prims\":[";
    for (size_t k = 0; k < RP.prims.size(); ++k) {
      const Prim& p = RP.prims[k];
      o << (k ? "," : "") << "{\"kind\":\"" << p.kind_name() << "\",\"chunk\":" << p.chunk << ",\"pc\":" << p.pc
        << ",\"recv_task\":" << p.recv_task << ",\"send_task\":" << p.send_task << ",\"src\":\""
        << buf_name(p.src_buf) << "\",\"dst\":\"" << buf_name(p.dst_buf) << "\",\"cta\":" << p.cta
        << ",\"lane\":" << p.lane << ",\"counter\":" << (p.has_counter ? "true" : "false")
        << ",\"rem\":\"" << buf_name(p.rem_buf) << "\",\"rem_out\":\"" << buf_name(p.rem_out) << "\",\"deps\":[";
      for (size_t d = 0; d < p.deps.size(); ++d) o << (d ? "," : "") << p.deps[d];
      o << "],\"ack_deps\":[";
      for (size_t d = 0; d < p.ack_deps.size(); ++d) o << (d ? "," : "") << p.ack_deps[d];
      o << "]}";
    }
    o << "]}";
  }
  o << "]}";
  return o.str();
}

}  // namespace resccl
