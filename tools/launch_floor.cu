// Launch and handoff floors on B200 (d8 overhead budget): what a collective kernel pays
// before any data moves.  Every number is the per-launch time of 20 launches captured in
// one CUDA graph and replayed (device clock, CUDA events), best of 5 replays.
//   empty   : an empty kernel, grid x threads, dynamic shared memory smem bytes
//   coop    : the same through cudaLaunchCooperativeKernel
//   chain   : a chain of `hops` cross-CTA handoffs: CTA h waits for flag h-1 (leader
//             polling ld.acquire.gpu), posts flag h; the last CTA's post ends the chain.
//             post variants: 0 fence.acq_rel.gpu + st.relaxed, 1 st.release.gpu,
//             2 red.release.gpu.add
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o launch_floor tools/launch_floor.cu
// ./launch_floor <grid> <threads> <smem KiB> <hops>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)
typedef unsigned long long u64;

__global__ void k_empty() {}

__device__ __forceinline__ u64 ld_acq(const u64* p) {
  u64 v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ u64 ld_rlx(const u64* p) {
  u64 v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// flags[h] is monotone across launches: launch e waits for flags[h-1] >= e+1
template <int POST, int POLL>
__global__ void k_chain(u64* flags, int hops, u64* epoch) {
  const int h = blockIdx.x;
  if (h >= hops || threadIdx.x != 0) return;
  const u64 e = ld_rlx(epoch) + 1;  // this launch's epoch (advanced by the last CTA)
  if (h > 0) {
    if (POLL == 0) {
      while (ld_acq(flags + h - 1) < e) {}
    } else {
      while (ld_rlx(flags + h - 1) < e) {}
      asm volatile("fence.acq_rel.gpu;" ::: "memory");
    }
  }
  if (POST == 0) {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(flags + h), "l"(e) : "memory");
  } else if (POST == 1) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(flags + h), "l"(e) : "memory");
  } else {
    asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(flags + h), "l"(1ull) : "memory");
  }
  if (h == hops - 1) *epoch = e;  // stream order publishes it to the next launch
}

template <class F>
float graph_us(F launch, cudaStream_t s) {
  cudaGraph_t g;
  cudaGraphExec_t ge;
  CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
  for (int i = 0; i < 20; ++i) launch();
  CK(cudaStreamEndCapture(s, &g));
  CK(cudaGraphInstantiate(&ge, g, 0));
  CK(cudaGraphLaunch(ge, s));
  CK(cudaStreamSynchronize(s));
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  float best = 1e30f;
  for (int r = 0; r < 5; ++r) {
    CK(cudaEventRecord(a, s));
    CK(cudaGraphLaunch(ge, s));
    CK(cudaEventRecord(b, s));
    CK(cudaEventSynchronize(b));
    float ms;
    CK(cudaEventElapsedTime(&ms, a, b));
    if (ms < best) best = ms;
  }
  CK(cudaGraphExecDestroy(ge));
  CK(cudaGraphDestroy(g));
  return best * 1e3f / 20;
}

int main(int argc, char** argv) {
  const int grid = argc > 1 ? atoi(argv[1]) : 96, nt = argc > 2 ? atoi(argv[2]) : 384;
  const int smem = (argc > 3 ? atoi(argv[3]) : 224) * 1024, hops = argc > 4 ? atoi(argv[4]) : 14;
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  CK(cudaFuncSetAttribute(k_empty, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  printf("{\"grid\": %d, \"threads\": %d, \"smem\": %d, \"hops\": %d", grid, nt, smem, hops);
  printf(", \"empty_nosmem_us\": %.2f", graph_us([&] { k_empty<<<grid, nt, 0, s>>>(); }, s));
  printf(", \"empty_us\": %.2f", graph_us([&] { k_empty<<<grid, nt, smem, s>>>(); }, s));
  printf(", \"coop_us\": %.2f", graph_us([&] {
           void* args[1] = {nullptr};
           CK(cudaLaunchCooperativeKernel((void*)k_empty, grid, nt, args, smem, s));
         }, s));
  u64 *flags, *epoch;
  CK(cudaMalloc(&flags, 4096 * 8));
  CK(cudaMalloc(&epoch, 8));
#define CHAIN(P, Q)                                                                              \
  {                                                                                            \
    CK(cudaMemset(flags, 0, 4096 * 8));                                                        \
    CK(cudaMemset(epoch, 0, 8));                                                               \
    CK(cudaFuncSetAttribute(k_chain<P, Q>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)); \
    const int g2 = grid > hops ? grid : hops;                                                  \
    printf(", \"chain_post%d_poll%d_us\": %.2f", P, Q,                                          \
           graph_us([&] { k_chain<P, Q><<<g2, nt, smem, s>>>(flags, hops, epoch); }, s));     \
  }
  CHAIN(0, 0) CHAIN(1, 0) CHAIN(0, 1) CHAIN(1, 1)
  // red.release counts launches: flags[h] == e after launch e as well
  CHAIN(2, 0)
  printf("}\n");
  return 0;
}
