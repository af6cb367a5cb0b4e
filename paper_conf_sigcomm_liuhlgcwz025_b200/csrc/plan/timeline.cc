// Wall-clock timeline simulation (timeline.h; Eq. 1, Eq. 5, Eq. 7 on active_l(t)).
#include "timeline.h"

#include <algorithm>
#include <cmath>
#include <map>
#include <set>
#include <sstream>
#include <tuple>

namespace resccl {

namespace {

struct Lane {
  int r, cta, lane, inst;
  const std::vector<int>* prog;
  int k = 0, j = 0, phase = 0;
  bool busy = false;
  double pen = 0, work = 0, start = 0;
  std::vector<std::tuple<int, int, int>> res;  // contended resources of the running invocation
};

}  // namespace

TimelineResult simulate_timeline(const Plan& P, const TimelineParams& tp) {
  const Ir& ir = P.ir;
  const int n_mb = tp.n_mb, K = tp.K, I = tp.instances;
  if (n_mb < 1 || K < 1 || I < 1) throw PlanError("timeline: n_mb, K and instances must be >= 1");
  if (!(tp.alpha >= 0 && tp.beta >= 0 && tp.gamma >= 0 && tp.c >= 0)) throw PlanError("timeline: negative cost");
  std::vector<Lane> lanes;
  for (int inst = 0; inst < I; ++inst)
    for (int r = 0; r < ir.nranks; ++r)
      for (int c = 0; c < (int)P.ranks[r].ctas.size(); ++c) {
        const auto& sl = P.ranks[r].ctas[c].first;
        const auto& rl = P.ranks[r].ctas[c].second;
        if (!sl.empty()) lanes.push_back({r, c, 0, inst, &sl});
        if (!rl.empty()) lanes.push_back({r, c, 1, inst, &rl});
      }
  using LK = std::tuple<int, int, int>;  // (src, dst, inst)
  std::map<std::tuple<int, int, int>, int> done;  // (rank, prim, inst) -> micro-batches finished
  std::map<LK, std::set<long>> produced;
  std::map<LK, long> credit;
  auto link = [&](int t, int inst) { return LK{ir.t[t].src, ir.t[t].dst, inst}; };
  auto pos_of = [&](int t, int j) { return (long)P.link_pos[t] * n_mb + j; };
  auto prim = [&](const Lane& L) -> const Prim& { return P.ranks[L.r].prims[(*L.prog)[L.k]]; };
  auto deps_ok = [&](const Lane& L, const Prim& pm) {
    for (int d : pm.deps)
      if (done[{L.r, d, L.inst}] < L.j + 1) return false;
    for (int d : pm.ack_deps) {
      int t = P.ranks[L.r].prims[d].send_task;
      if (credit[link(t, L.inst)] < pos_of(t, L.j) + 1) return false;
    }
    return true;
  };
  auto send_ok = [&](const Lane& L, const Prim& pm) {
    if (!(pm.flags & kSend)) return true;
    long pos = pos_of(pm.send_task, L.j);
    long cr = credit[link(pm.send_task, L.inst)];
    if (!(pm.flags & kDirect)) return pos < cr + K;
    if (pm.flags & kSendPull) return true;
    return cr >= pos + 1;
  };
  auto is_push_recv = [](const Prim& pm) {
    return (pm.flags & kDirect) && (pm.flags & kRecv) && !(pm.flags & kPull);
  };
  auto enabled = [&](Lane& L) {
    if (L.busy || L.k >= (int)L.prog->size()) return false;
    const Prim& pm = prim(L);
    if (pm.flags & kCopy) return true;
    if (is_push_recv(pm) && L.phase == 1)
      return produced[link(pm.recv_task, L.inst)].count(pos_of(pm.recv_task, L.j)) > 0 && send_ok(L, pm);
    if (!deps_ok(L, pm)) return false;
    if (is_push_recv(pm)) return true;
    if (pm.flags & kRecv)
      if (!produced[link(pm.recv_task, L.inst)].count(pos_of(pm.recv_task, L.j))) return false;
    return send_ok(L, pm);
  };
  // effects of a finished invocation (the plan check's blocking semantics)
  auto finish = [&](Lane& L) {
    int pid = (*L.prog)[L.k];
    const Prim& pm = P.ranks[L.r].prims[pid];
    const bool direct = pm.flags & kDirect, pull = pm.flags & kPull;
    L.phase = 0;
    if (pm.recv_task >= 0) {
      auto key = link(pm.recv_task, L.inst);
      long pos = pos_of(pm.recv_task, L.j);
      produced[key].erase(pos);
      if (!direct) credit[key] += 1;
      else if (pull) credit[key] = std::max(credit[key], pos + 1);
    }
    if (pm.send_task >= 0) produced[link(pm.send_task, L.inst)].insert(pos_of(pm.send_task, L.j));
    if (!(pm.flags & kCopy)) done[{L.r, pid, L.inst}] = L.j + 1;
    L.j++;
    if (L.j >= ((pm.flags & kCopy) ? 1 : n_mb)) {
      L.k++;
      L.j = 0;
    }
  };
  // contended resources of an invocation: the links it moves data over
  auto resources = [&](const Prim& pm) {
    std::vector<std::tuple<int, int, int>> res;
    auto add = [&](int t) {
      const Transfer& x = ir.t[t];
      if (P.model == LinkModel::Pair) {
        res.emplace_back(0, x.src, x.dst);
      } else {
        res.emplace_back(1, x.src, -1);  // egress port of the sender
        res.emplace_back(2, x.dst, -1);  // ingress port of the receiver
      }
    };
    const bool direct = pm.flags & kDirect;
    if ((pm.flags & kSend) && !(direct && (pm.flags & kSendPull))) add(pm.send_task);
    if (direct && (pm.flags & kRecv) && (pm.flags & kPull)) add(pm.recv_task);
    return res;
  };

  TimelineResult R;
  R.conns.assign(ir.nranks, {});
  R.conn_active.assign(ir.nranks, {});
  std::vector<std::map<std::pair<int, int>, int>> conn_idx(ir.nranks);
  auto conn_of = [&](int r, int peer, int dir) {
    auto it = conn_idx[r].find({peer, dir});
    if (it != conn_idx[r].end()) return it->second;
    int id = (int)R.conns[r].size();
    conn_idx[r][{peer, dir}] = id;
    R.conns[r].push_back({peer, dir});
    R.conn_active[r].push_back({});
    return id;
  };
  R.lane_busy.assign(lanes.size(), 0.0);
  std::map<std::tuple<int, int, int>, int> load;  // resource -> invocations in their work phase
  double t = 0;
  const double tiny = 1e-15;
  auto z_of = [&](const Lane& L) {
    int z = 1;
    for (auto& x : L.res) z = std::max(z, load[x]);
    return z;
  };
  for (;;) {
    // (a) instantaneous "writable" posts, to a fixpoint
    bool changed = true;
    while (changed) {
      changed = false;
      for (auto& L : lanes) {
        if (!enabled(L)) continue;
        const Prim& pm = prim(L);
        if (is_push_recv(pm) && L.phase == 0) {
          auto key = link(pm.recv_task, L.inst);
          credit[key] = std::max(credit[key], pos_of(pm.recv_task, L.j) + 1);
          L.phase = 1;
          changed = true;
        }
      }
    }
    // (b) every enabled invocation starts at time t; simultaneous starters on a link see
    // the same contention z (Eq. 1's penalty is symmetric)
    std::vector<size_t> starters;
    std::map<std::tuple<int, int, int>, int> starting;
    for (size_t i = 0; i < lanes.size(); ++i) {
      Lane& L = lanes[i];
      if (!enabled(L)) continue;
      starters.push_back(i);
      L.res = resources(prim(L));
      for (auto& x : L.res) starting[x]++;
    }
    for (size_t i : starters) {
      Lane& L = lanes[i];
      L.busy = true;
      L.start = t;
      L.work = tp.alpha + (L.res.empty() ? 0.0 : tp.c * tp.beta);
      int z0 = 1;
      for (auto& x : L.res) z0 = std::max(z0, load[x] + starting[x]);
      L.pen = tp.gamma * (double)(z0 - 1) / (double)n_mb;
    }
    for (size_t i : starters)
      if (lanes[i].pen <= 0)
        for (auto& x : lanes[i].res) load[x]++;
    bool any = false, all_done = true;
    for (auto& L : lanes) {
      any = any || L.busy;
      all_done = all_done && L.k >= (int)L.prog->size();
    }
    if (all_done) break;
    if (!any) throw PlanError("timeline: the plan deadlocks");
    // next event: a penalty ends or an invocation's work ends
    double dt = INFINITY;
    for (auto& L : lanes) {
      if (!L.busy) continue;
      if (L.pen > 0) dt = std::min(dt, L.pen);
      else dt = std::min(dt, L.work * z_of(L));
    }
    std::vector<int> zs(lanes.size(), 1);
    for (size_t i = 0; i < lanes.size(); ++i)
      if (lanes[i].busy && lanes[i].pen <= 0) {
        zs[i] = z_of(lanes[i]);
        R.max_z = std::max(R.max_z, (double)zs[i]);
      }
    t += dt;
    for (size_t i = 0; i < lanes.size(); ++i) {
      Lane& L = lanes[i];
      if (!L.busy) continue;
      if (L.pen > 0) {
        L.pen -= dt;
        if (L.pen <= tiny * std::max(1.0, t)) {
          L.pen = 0;
          for (auto& x : L.res) load[x]++;
        }
        continue;
      }
      L.work -= dt / zs[i];
    }
    for (size_t i = 0; i < lanes.size(); ++i) {
      Lane& L = lanes[i];
      if (!L.busy || L.pen > 0 || L.work > tiny * std::max(1.0, t)) continue;
      const Prim& pm = prim(L);
      for (auto& x : L.res) load[x]--;
      L.busy = false;
      R.lane_busy[i] += t - L.start;
      if (L.inst == 0) {
        if (pm.send_task >= 0) R.conn_active[L.r][conn_of(L.r, ir.t[pm.send_task].dst, 0)].push_back({L.start, t});
        if (pm.recv_task >= 0) R.conn_active[L.r][conn_of(L.r, ir.t[pm.recv_task].src, 1)].push_back({L.start, t});
      }
      finish(L);
    }
  }
  R.makespan = t;
  // Eq. 7 on the wall clock: merge connections of one direction whose activity never
  // overlaps, greedily in order of first activity
  R.merged_send.assign(ir.nranks, 0);
  R.merged_recv.assign(ir.nranks, 0);
  for (int r = 0; r < ir.nranks; ++r) {
    for (int dir = 0; dir < 2; ++dir) {
      std::vector<int> ids;
      for (int c = 0; c < (int)R.conns[r].size(); ++c)
        if (R.conns[r][c].second == dir && !R.conn_active[r][c].empty()) ids.push_back(c);
      auto first = [&](int c) {
        double f = INFINITY;
        for (auto& x : R.conn_active[r][c]) f = std::min(f, x.first);
        return f;
      };
      std::sort(ids.begin(), ids.end(), [&](int a, int b) {
        return std::make_pair(first(a), R.conns[r][a].first) < std::make_pair(first(b), R.conns[r][b].first);
      });
      std::vector<std::vector<std::pair<double, double>>> groups;
      for (int c : ids) {
        const auto& iv = R.conn_active[r][c];
        bool placed = false;
        for (auto& g : groups) {
          bool overlap = false;
          for (auto& a : iv) {
            for (auto& b : g)
              if (a.first < b.second && b.first < a.second) {
                overlap = true;
                break;
              }
            if (overlap) break;
          }
          if (!overlap) {
            g.insert(g.end(), iv.begin(), iv.end());
            placed = true;
            break;
          }
        }
        if (!placed) groups.push_back(iv);
      }
      (dir ? R.merged_recv : R.merged_send)[r] = (int)groups.size();
    }
  }
  return R;
}

std::string timeline_json(const Plan& P, const TimelineParams& tp, const TimelineResult& R) {
  std::ostringstream o;
  o.precision(17);
  const size_t nl = R.lane_busy.size();
  double busy = 0, max_idle = 0;
  for (double b : R.lane_busy) {
    busy += b;
    max_idle = std::max(max_idle, R.makespan > 0 ? 1.0 - b / R.makespan : 0.0);
  }
  const double comm = nl && R.makespan > 0 ? busy / (nl * R.makespan) : 0.0;
  o << "{\"makespan_s\":" << R.makespan << ",\"alpha\":" << tp.alpha << ",\"beta\":" << tp.beta
    << ",\"gamma\":" << tp.gamma << ",\"c\":" << tp.c << ",\"n_mb\":" << tp.n_mb << ",\"K\":" << tp.K
    << ",\"instances\":" << tp.instances << ",\"lanes\":" << nl << ",\"comm_time\":" << comm
    << ",\"avg_idle\":" << (nl ? 1.0 - comm : 0.0) << ",\"max_idle\":" << max_idle << ",\"max_z\":" << R.max_z
    << ",\"ranks\":[";
  for (int r = 0; r < P.ir.nranks; ++r) {
    o << (r ? "," : "") << "{\"merged_send\":" << R.merged_send[r] << ",\"merged_recv\":" << R.merged_recv[r]
      << ",\"pidx_send\":" << P.ranks[r].send_groups.size() << ",\"pidx_recv\":" << P.ranks[r].recv_groups.size()
      << ",\"conns\":[";
    for (size_t c = 0; c < R.conns[r].size(); ++c) {
      o << (c ? "," : "") << "{\"peer\":" << R.conns[r][c].first << ",\"dir\":\""
        << (R.conns[r][c].second ? "recv" : "send") << "\",\"active\":[";
      // union of the intervals
      auto iv = R.conn_active[r][c];
      std::sort(iv.begin(), iv.end());
      std::vector<std::pair<double, double>> u;
      for (auto& x : iv) {
        if (!u.empty() && x.first <= u.back().second) u.back().second = std::max(u.back().second, x.second);
        else u.push_back(x);
      }
      for (size_t k = 0; k < u.size(); ++k) o << (k ? "," : "") << "[" << u[k].first << "," << u[k].second << "]";
      o << "]}";
    }
    o << "]}";
  }
  o << "]}";
  return o.str();
}

}  // namespace resccl
