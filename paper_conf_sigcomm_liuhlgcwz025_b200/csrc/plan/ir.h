// ResCCL algorithm IR: the ResCCLang transfer model (§4.2;
// BNF Fig. 14) and the built-in algorithm generators.
//
// An algorithm is a list of Transfer(srcRank, dstRank, step, chunkId, opType),
// opType in {recv, rrc}.  Every rank's DataBuffer has nChunks = nRanks chunks and
// <Rank, ChunkId> is unique.  The IR carries no channels, TB hints
// or protocol: those are decided by the planner.
#pragma once

#include <cstdint>
#include <map>
#include <stdexcept>
#include <string>
#include <vector>

namespace resccl {

struct PlanError : std::runtime_error {
  using std::runtime_error::runtime_error;
};

enum class Op : uint8_t { Recv = 0, Rrc = 1 };
enum class Coll : uint8_t { AllGather = 0, ReduceScatter = 1, AllReduce = 2 };

const char* coll_name(Coll c);
Coll coll_from_name(const std::string& s);

struct Transfer {
  int src, dst, step, chunk;
  Op op;
  bool operator==(const Transfer& o) const {
    return src == o.src && dst == o.dst && step == o.step && chunk == o.chunk && op == o.op;
  }
};

struct Ir {
  std::string name;
  Coll coll = Coll::AllReduce;
  int nranks = 0;
  int nchunks = 0;
  int nwarps = 16;
  std::map<std::string, std::string> extra;  // header keys beyond the five above
  std::vector<Transfer> t;

  std::string to_text() const;
  long get_int(const std::string& key, long dflt) const;
};

// Text format (one transfer per line):
//   algo name=ring coll=allreduce nranks=8 nchunks=8 nwarps=16 [key=value ...]
//   t <src> <dst> <step> <chunk> <recv|rrc>
// '#' starts a comment.  Throws PlanError on malformed input.
Ir parse_ir(const std::string& text);

// ---- generators -----------------------------------------------------------
// ring AG: Fig. 5a listing; ring RS / AR: reading R10 (AR = RS then
// AG).
Ir gen_ring(Coll coll, int n);
// Double binary tree (NCCL's btree + mirrored tree), reading R11.
Ir gen_dbt_allreduce(int n);
// Hierarchical mesh AllReduce: Fig. 16 listing.
Ir gen_hm_allreduce(int n_nodes, int g);
// Hierarchical mesh AllGather: App. A, reading R12.
Ir gen_hm_allgather(int n_nodes, int g);
// Seeded TACCL-style trees (reading R13).
Ir gen_synth(Coll coll, int n, uint64_t seed, int fanout);

// name in {ring, dbt, hm, synth}; opts: g (GPUs per node), seed, fanout.
Ir generate(const std::string& name, Coll coll, int n, const std::map<std::string, long>& opts);

uint64_t splitmix64(uint64_t x);

// ResCCLang front end (BNF Fig. 14): executes a `def ResCCLAlgo(...):`
// program (e.g. the Fig. 16 listing) and returns its transfer IR.  Throws PlanError.
Ir parse_rescclang(const std::string& program);

}  // namespace resccl
