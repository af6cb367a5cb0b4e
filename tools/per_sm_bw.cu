// Per-SM memory-throughput ceilings on B200 (calibration for the lane engine):
// one CTA per SM on `nb` SMs streams its own contiguous range of HBM and we report
// (bytes read + bytes written) / time per SM.
//   mode 0: LDG/STG copy, U 16-byte vectors in flight per thread
//   mode 1: LDG/STG bf16 reduce D = A + B (fp32 combine, RNE), U vectors per operand
//   mode 2: TMA bulk copy global -> smem -> global, one leader thread, S stages of T bytes
//   mode 3: TMA reduce: leader streams A and B tiles in, the other warps combine in smem,
//           the leader bulk-stores D
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o per_sm_bw tools/per_sm_bw.cu
// ./per_sm_bw <mode> <nb> <threads> <U|S> <T bytes> <MiB per CTA>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include <cuda_bf16.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

struct V4 { unsigned x, y, z, w; };
__device__ __forceinline__ V4 ldg(const V4* p) {
  V4 v;
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ void stg(V4* p, V4 v) {
  asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ unsigned addbf(unsigned a, unsigned b) {
  float lo = __uint_as_float(a << 16) + __uint_as_float(b << 16);
  float hi = __uint_as_float(a & 0xffff0000u) + __uint_as_float(b & 0xffff0000u);
  unsigned r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}
__device__ __forceinline__ V4 addv(V4 a, V4 b) { return V4{addbf(a.x, b.x), addbf(a.y, b.y), addbf(a.z, b.z), addbf(a.w, b.w)}; }

template <int U>
__global__ void k_ldst(const V4* A, const V4* B, V4* D, long long nvec_per_cta, int reduce) {
  const long long base = blockIdx.x * nvec_per_cta;
  const int nt = blockDim.x;
  for (long long i = threadIdx.x; i < nvec_per_cta; i += (long long)U * nt) {
    V4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      long long k = i + (long long)u * nt;
      if (k < nvec_per_cta) { a[u] = ldg(A + base + k); if (reduce) b[u] = ldg(B + base + k); }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      long long k = i + (long long)u * nt;
      if (k < nvec_per_cta) stg(D + base + k, reduce ? addv(a[u], b[u]) : a[u]);
    }
  }
}

__device__ __forceinline__ unsigned sa(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(unsigned b, unsigned c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(c)); }
__device__ __forceinline__ void mb_tx(unsigned b, unsigned n) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(n) : "memory"); }
__device__ __forceinline__ void mb_arrive(unsigned b) { asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(b) : "memory"); }
__device__ __forceinline__ void mb_wait(unsigned b, unsigned par) {
  asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(b), "r"(par) : "memory");
}
__device__ __forceinline__ void tload(unsigned dst, const void* src, unsigned n, unsigned bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst), "l"(src), "r"(n), "r"(bar) : "memory");
}
__device__ __forceinline__ void tstore(void* dst, unsigned src, unsigned n) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src), "r"(n) : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
template <int N> __device__ __forceinline__ void wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }

// S stages, store lag L = S/2: before loading tile t into stage t%S, the store of tile t-S
// (issued S-L iterations ago... ) must have read the stage out.
template <int S>
__global__ void k_tma(const char* A, const char* B, char* D, long long bytes_per_cta, int T, int reduce) {
  extern __shared__ __align__(128) char sm[];
  __shared__ __align__(8) unsigned long long full[S], comp[S];
  const long long base = blockIdx.x * bytes_per_cta;
  const int ntile = (int)(bytes_per_cta / T);
  char* st = sm;  // stage s: A at s*2T, B at s*2T+T
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) { mb_init(sa(&full[s]), 1); mb_init(sa(&comp[s]), (blockDim.x - 32) / 32); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  constexpr int L = S / 2;
  if (threadIdx.x == 0) {
    for (int t = 0; t < ntile + L; ++t) {
      if (t < ntile) {
        const int s = t % S;
        if (t >= S) wait_read<S - L - 1>();
        const unsigned bar = sa(&full[s]);
        mb_tx(bar, reduce ? 2 * T : T);
        tload(sa(st + (size_t)s * 2 * T), A + base + (long long)t * T, T, bar);
        if (reduce) tload(sa(st + (size_t)s * 2 * T + T), B + base + (long long)t * T, T, bar);
      }
      const int u = t - L;
      if (u >= 0) {
        const int s = u % S;
        const unsigned par = (u / S) & 1;
        if (reduce) mb_wait(sa(&comp[s]), par); else mb_wait(sa(&full[s]), par);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        tstore(D + base + (long long)u * T, sa(st + (size_t)s * 2 * T), T);
      }
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  } else if (threadIdx.x >= 32 && reduce) {
    const int ct = threadIdx.x - 32, nct = blockDim.x - 32;
    for (int u = 0; u < ntile; ++u) {
      const int s = u % S;
      mb_wait(sa(&full[s]), (u / S) & 1);
      const unsigned a = sa(st + (size_t)s * 2 * T);
      for (int i = ct; i < T / 16; i += nct) {
        V4 x, y;
        asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(x.x), "=r"(x.y), "=r"(x.z), "=r"(x.w) : "r"(a + 16 * i));
        asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(y.x), "=r"(y.y), "=r"(y.z), "=r"(y.w) : "r"(a + T + 16 * i));
        V4 z = addv(x, y);
        asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a + 16 * i), "r"(z.x), "r"(z.y), "r"(z.z), "r"(z.w) : "memory");
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if ((threadIdx.x & 31) == 0) mb_arrive(sa(&comp[s]));
    }
  }
}

int main(int argc, char** argv) {
  if (argc < 7) { printf("usage: mode nb threads U|S T MiB\n"); return 1; }
  const int mode = atoi(argv[1]), nb = atoi(argv[2]), nt = atoi(argv[3]), US = atoi(argv[4]), T = atoi(argv[5]);
  const long long per = (long long)(atof(argv[6]) * (1 << 20));
  const size_t tot = (size_t)per * nb;
  char *A, *B, *D;
  CK(cudaMalloc(&A, tot)); CK(cudaMalloc(&B, tot)); CK(cudaMalloc(&D, tot));
  CK(cudaMemset(A, 1, tot)); CK(cudaMemset(B, 2, tot));
  const int reduce = (mode == 1 || mode == 3);
  auto run = [&]() {
    if (mode <= 1) {
      const long long nv = per / 16;
      if (US == 2) k_ldst<2><<<nb, nt>>>((V4*)A, (V4*)B, (V4*)D, nv, reduce);
      else if (US == 4) k_ldst<4><<<nb, nt>>>((V4*)A, (V4*)B, (V4*)D, nv, reduce);
      else if (US == 8) k_ldst<8><<<nb, nt>>>((V4*)A, (V4*)B, (V4*)D, nv, reduce);
      else k_ldst<16><<<nb, nt>>>((V4*)A, (V4*)B, (V4*)D, nv, reduce);
    } else {
      const size_t smem = (size_t)US * 2 * T;
#define L_(S_) do { CK(cudaFuncSetAttribute(k_tma<S_>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)); \
        k_tma<S_><<<nb, nt, smem>>>(A, B, D, per, T, reduce); } while (0)
      switch (US) { case 2: L_(2); break; case 4: L_(4); break; case 6: L_(6); break; case 8: L_(8); break; case 12: L_(12); break; default: L_(16); }
    }
  };
  run();
  CK(cudaGetLastError());  // e.g. too many registers for the block size: no timing line
  CK(cudaDeviceSynchronize());
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int it = 10;
  cudaEventRecord(e0);
  for (int i = 0; i < it; ++i) run();
  cudaEventRecord(e1);
  CK(cudaEventSynchronize(e1));
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  ms /= it;
  const double bytes = (double)tot * (reduce ? 3 : 2);
  printf("{\"mode\": %d, \"nb\": %d, \"threads\": %d, \"US\": %d, \"T\": %d, \"MiB_per_cta\": %g, \"us\": %.1f, \"total_gbs\": %.1f, \"per_sm_gbs\": %.1f}\n",
         mode, nb, nt, US, T, per / 1048576.0, ms * 1e3, bytes / ms / 1e6, bytes / ms / 1e6 / nb);
  return 0;
}
