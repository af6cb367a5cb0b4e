// Oracle: C++17 fast schedule replay for full-size buffers.
// TEST INFRASTRUCTURE ONLY -- called from tests/ and bench.py's cpu_baseline / --impl
// reference legs through oracle/fastreplay.py.  No CUDA header, no code shared with the
// product (paper_conf_sigcomm_liuhlgcwz025_b200/): it has its own IR reader and its own
// element arithmetic.
//
// What it computes: the algorithm's transfers ("transfer(src,
// dst, step, chunk, recv|rrc)") applied literally in step order to the locations
// <rank, chunk> (reading R1: conflicts at a location are ordered by step, no two
// conflicting transfers share a step), i.e. the association order every lowering of the
// IR realises (pinned: replay.dataflow_values == replay.replay, tests/test_oracle_pins_r2):
//   recv:  <dst, c> := <src, c>
//   rrc:   <dst, c> := <dst, c> (+) <src, c>         (local (+) incoming, reading R8)
// (+) per element: int32 two's-complement wrap; fp32 binary32 add; bf16 / fp16 widened
// to binary32, added, rounded to nearest even back to the storage type (R8).  Only sum.
//
// Chunk layout (reading R6): AllReduce chunk c = elements [c*C, c*C + len_c) with
// C = ceil(count / N) rounded up to 256 bytes; AllGather / ReduceScatter chunk c = rank
// c's segment of `count` elements.  Every element of a chunk follows the same transfers
// and chunks never interact (no cross-chunk DAG edges), so the work splits into
// independent (chunk, element block) tasks run by `threads` std::threads; each task
// replays the chunk's whole step sequence on its block.
#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cstring>
#include <sstream>
#include <string>
#include <thread>
#include <vector>

namespace {

struct Xfer {
  int src, dst, step, chunk;
  bool rrc;
};

enum { DInt32 = 0, DFloat32 = 1, DFloat16 = 2, DBfloat16 = 3 };
enum { AllGather = 0, ReduceScatter = 1, AllReduce = 2 };

bool parse(const char* text, int* coll, int* nranks, std::vector<Xfer>* xs) {
  std::istringstream is(text);
  std::string line;
  *coll = -1;
  *nranks = 0;
  while (std::getline(is, line)) {
    std::istringstream ls(line);
    std::string w;
    if (!(ls >> w)) continue;
    if (w == "algo") {
      while (ls >> w) {
        auto e = w.find('=');
        if (e == std::string::npos) continue;
        std::string k = w.substr(0, e), v = w.substr(e + 1);
        if (k == "coll") *coll = v == "allgather" ? AllGather : v == "reducescatter" ? ReduceScatter
                                 : v == "allreduce" ? AllReduce : -1;
        if (k == "nranks") *nranks = std::stoi(v);
      }
    } else if (w == "t") {
      Xfer x;
      std::string op;
      if (!(ls >> x.src >> x.dst >> x.step >> x.chunk >> op)) return false;
      if (op != "recv" && op != "rrc") return false;
      x.rrc = op == "rrc";
      xs->push_back(x);
    }
  }
  return *coll >= 0 && *nranks > 0;
}

inline float f32_of_bits(uint32_t u) {
  float f;
  std::memcpy(&f, &u, 4);
  return f;
}
inline uint32_t bits_of_f32(float f) {
  uint32_t u;
  std::memcpy(&u, &f, 4);
  return u;
}
inline float bf16_to_f32(uint16_t h) { return f32_of_bits((uint32_t)h << 16); }
inline uint16_t f32_to_bf16(float f) {  // round to nearest even (no NaN inputs)
  const uint32_t u = bits_of_f32(f);
  return (uint16_t)((u + 0x7FFFu + ((u >> 16) & 1u)) >> 16);
}
inline float f16_to_f32(uint16_t h) {
  const uint32_t s = (uint32_t)(h & 0x8000u) << 16, e = (h >> 10) & 0x1Fu, m = h & 0x3FFu;
  if (e == 0) {  // zero / subnormal: m * 2^-24 (exact in binary32)
    const float v = (float)m * 5.9604644775390625e-08f;
    return s ? -v : v;
  }
  if (e == 31) return f32_of_bits(s | 0x7F800000u | (m << 13));
  return f32_of_bits(s | ((e - 15 + 127) << 23) | (m << 13));
}
inline uint16_t f32_to_f16(float f) {  // round to nearest even, subnormals kept
  const uint32_t x = bits_of_f32(f);
  const uint16_t sign = (uint16_t)((x >> 16) & 0x8000u);
  const uint32_t ax = x & 0x7FFFFFFFu;
  if (ax >= 0x7F800000u) return sign | 0x7C00u | (ax > 0x7F800000u ? 0x200u : 0u);
  if (ax >= 0x477FF000u) return sign | 0x7C00u;  // >= 65520 rounds to infinity
  if (ax < 0x38800000u) {                         // below 2^-14: subnormal quantum 2^-24
    const uint32_t e = ax >> 23;
    if (e < 102) return sign;                      // < 2^-25: rounds to zero
    const uint32_t mant = (ax & 0x7FFFFFu) | 0x800000u;
    const uint32_t shift = 126 - e;                // value = mant * 2^(e-150); units of 2^-24
    uint32_t q = mant >> shift;
    const uint32_t rem = mant & ((1u << shift) - 1u), half = 1u << (shift - 1);
    if (rem > half || (rem == half && (q & 1u))) ++q;
    return sign | (uint16_t)q;
  }
  uint32_t h = ((((ax >> 23) - 112u) << 10) | ((ax & 0x7FFFFFu) >> 13));
  const uint32_t rem = ax & 0x1FFFu;
  if (rem > 0x1000u || (rem == 0x1000u && (h & 1u))) ++h;
  return sign | (uint16_t)h;
}

template <int DT>
void combine(void* dst, const void* src, int64_t n) {
  if (DT == DInt32) {
    auto* d = (uint32_t*)dst;
    auto* s = (const uint32_t*)src;
    for (int64_t i = 0; i < n; ++i) d[i] = d[i] + s[i];
  } else if (DT == DFloat32) {
    auto* d = (float*)dst;
    auto* s = (const float*)src;
    for (int64_t i = 0; i < n; ++i) d[i] = d[i] + s[i];
  } else if (DT == DBfloat16) {
    auto* d = (uint16_t*)dst;
    auto* s = (const uint16_t*)src;
    for (int64_t i = 0; i < n; ++i) d[i] = f32_to_bf16(bf16_to_f32(d[i]) + bf16_to_f32(s[i]));
  } else {
    auto* d = (uint16_t*)dst;
    auto* s = (const uint16_t*)src;
    for (int64_t i = 0; i < n; ++i) d[i] = f32_to_f16(f16_to_f32(d[i]) + f16_to_f32(s[i]));
  }
}

void combine_dt(int dt, void* d, const void* s, int64_t n) {
  switch (dt) {
    case DInt32: combine<DInt32>(d, s, n); break;
    case DFloat32: combine<DFloat32>(d, s, n); break;
    case DFloat16: combine<DFloat16>(d, s, n); break;
    default: combine<DBfloat16>(d, s, n); break;
  }
}

}  // namespace

extern "C" {

// Replays `ir_text` on full host buffers.  send[r] / recv[r]: rank r's send and receive
// buffers in the collective's layout (AR: count elements each; AG: send count, recv
// N*count; RS: send N*count, recv count).  `work` (RS only; else may be NULL): N
// buffers of N*count elements the replay may use as the ranks' chunk locations.
// Returns 0 on success, 1 on a malformed IR, 2 on a bad argument.
int oracle_fast_replay(const char* ir_text, int dtype, const void* const* send, void* const* recv,
                       void* const* work, long long count, int threads) {
  int coll, N;
  std::vector<Xfer> xs;
  if (!ir_text || !parse(ir_text, &coll, &N, &xs)) return 1;
  if (dtype < 0 || dtype > 3 || count < 0 || threads < 1) return 2;
  const int64_t e = (dtype == DInt32 || dtype == DFloat32) ? 4 : 2;
  for (auto& x : xs)
    if (x.src < 0 || x.src >= N || x.dst < 0 || x.dst >= N || x.chunk < 0 || x.chunk >= N) return 1;
  std::stable_sort(xs.begin(), xs.end(), [](const Xfer& a, const Xfer& b) { return a.step < b.step; });
  // locations: loc[r] = base of rank r's chunk array, chunk c at c * C elements
  int64_t C = count;
  std::vector<char*> loc(N);
  std::vector<int64_t> len(N, count);
  if (coll == AllReduce) {
    const int64_t q = 256 / e;
    C = count ? ((count + N - 1) / N + q - 1) / q * q : 0;
    for (int c = 0; c < N; ++c) len[c] = std::max<int64_t>(0, std::min<int64_t>(C, count - (int64_t)c * C));
    for (int r = 0; r < N; ++r) {
      loc[r] = (char*)recv[r];
      if (recv[r] != send[r]) std::memcpy(recv[r], send[r], (size_t)(count * e));
    }
  } else if (coll == AllGather) {
    for (int r = 0; r < N; ++r) {
      loc[r] = (char*)recv[r];
      char* own = (char*)recv[r] + (size_t)r * count * e;
      if (own != send[r]) std::memmove(own, send[r], (size_t)(count * e));
    }
  } else {
    if (!work) return 2;
    for (int r = 0; r < N; ++r) {
      loc[r] = (char*)work[r];
      std::memcpy(work[r], send[r], (size_t)(N * count * e));
    }
  }
  // tasks: (chunk, element block)
  const int64_t B = 1 << 15;
  std::vector<std::pair<int, int64_t>> tasks;
  for (int c = 0; c < N; ++c)
    for (int64_t lo = 0; lo < len[c]; lo += B) tasks.push_back({c, lo});
  std::vector<std::vector<const Xfer*>> of_chunk(N);
  for (auto& x : xs) of_chunk[x.chunk].push_back(&x);
  std::atomic<size_t> next(0);
  auto worker = [&]() {
    for (size_t t; (t = next.fetch_add(1)) < tasks.size();) {
      const int c = tasks[t].first;
      const int64_t lo = tasks[t].second, n = std::min<int64_t>(B, len[c] - lo);
      const int64_t off = ((int64_t)c * C + lo) * e;
      for (const Xfer* x : of_chunk[c]) {
        char* d = loc[x->dst] + off;
        const char* s = loc[x->src] + off;
        if (x->rrc) combine_dt(dtype, d, s, n);
        else std::memcpy(d, s, (size_t)(n * e));
      }
    }
  };
  std::vector<std::thread> pool;
  for (int i = 1; i < threads; ++i) pool.emplace_back(worker);
  worker();
  for (auto& th : pool) th.join();
  if (coll == ReduceScatter)
    for (int r = 0; r < N; ++r)
      std::memcpy(recv[r], (char*)work[r] + (size_t)r * count * e, (size_t)(count * e));
  return 0;
}

}  // extern "C"
