// Probe (f3 prerequisite): can this box create an NVLink-SHARP multicast object and run
// multimem.ld_reduce / multimem.st on it?  Prints one JSON line per driver step.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o build/nvls_probe tools/nvls_probe.cu -lcuda
//   build/nvls_probe [twice]   (twice: try adding the same device to the object twice)
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdio.h>
#define CK(x)                                                                  \
  do {                                                                         \
    CUresult r_ = (x);                                                         \
    const char* s_ = 0;                                                        \
    cuGetErrorName(r_, &s_);                                                   \
    printf("{\"step\": \"%s\", \"result\": \"%s\"}\n", #x, s_);                \
    if (r_ != CUDA_SUCCESS) return 1;                                          \
  } while (0)

__global__ void k(float* mc, float* uc, int n, float* out) {
  int i = threadIdx.x * 4;
  if (i >= n) return;
  float4 v = make_float4(1.f + i, 2.f + i, 3.f + i, 4.f + i);
  asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(mc + i), "f"(v.x), "f"(v.y),
               "f"(v.z), "f"(v.w)
               : "memory");
  asm volatile("fence.proxy.alias;" ::: "memory");
  __syncthreads();
  float a, b, c, d;
  asm volatile("multimem.ld_reduce.relaxed.sys.global.add.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(a), "=f"(b), "=f"(c), "=f"(d)
               : "l"(mc + i)
               : "memory");
  out[i] = a;
  out[i + 1] = b;
  out[i + 2] = c;
  out[i + 3] = d;
  out[n + i] = uc[i];
  out[n + i + 1] = uc[i + 1];
  out[n + i + 2] = uc[i + 2];
  out[n + i + 3] = uc[i + 3];
}

int main(int argc, char** argv) {
  int twice = argc > 1;
  CK(cuInit(0));
  CUdevice dev;
  CK(cuDeviceGet(&dev, 0));
  CUcontext ctx;
  CK(cuDevicePrimaryCtxRetain(&ctx, dev));
  CK(cuCtxSetCurrent(ctx));
  int sup = 0, fab = 0;
  cuDeviceGetAttribute(&sup, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev);
  cuDeviceGetAttribute(&fab, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, dev);
  printf("{\"multicast_supported\": %d, \"fabric_handles\": %d}\n", sup, fab);
  size_t sz = 2 << 20;
  {  // which (handle type, numDevices, size) combinations does cuMulticastCreate accept?
    const CUmemAllocationHandleType ht[3] = {CU_MEM_HANDLE_TYPE_NONE, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR,
                                             CU_MEM_HANDLE_TYPE_FABRIC};
    for (int h = 0; h < 3; ++h)
      for (int nd = 1; nd <= 2; ++nd)
        for (size_t s2 = 2 << 20; s2 <= (64u << 20); s2 *= 32) {
          CUmulticastObjectProp q = {};
          q.numDevices = nd;
          q.size = s2;
          q.handleTypes = ht[h];
          CUmemGenericAllocationHandle m2;
          CUresult r = cuMulticastCreate(&m2, &q);
          const char* nm = 0;
          cuGetErrorName(r, &nm);
          printf("{\"create_handle\": %d, \"numDevices\": %d, \"size\": %zu, \"result\": \"%s\"}\n", (int)ht[h], nd, s2, nm);
          if (r == CUDA_SUCCESS) {
            CUresult r2 = cuMulticastAddDevice(m2, dev);
            cuGetErrorName(r2, &nm);
            printf("{\"add_device\": \"%s\"}\n", nm);
            cuMemRelease(m2);
          }
        }
  }
  CUmulticastObjectProp mp = {};
  mp.numDevices = twice ? 2 : 1;
  mp.size = sz;
  mp.handleTypes = CU_MEM_HANDLE_TYPE_FABRIC;
  size_t g = 0;
  CK(cuMulticastGetGranularity(&g, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED));
  printf("{\"granularity\": %zu}\n", g);
  CUmemGenericAllocationHandle mc;
  CK(cuMulticastCreate(&mc, &mp));
  CK(cuMulticastAddDevice(mc, dev));
  if (twice) CK(cuMulticastAddDevice(mc, dev));
  CUmemAllocationProp ap = {};
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = 0;
  CUmemGenericAllocationHandle mem;
  CK(cuMemCreate(&mem, sz, &ap, 0));
  CK(cuMulticastBindMem(mc, 0, mem, 0, sz, 0));
  CUdeviceptr va_mc, va_uc;
  CK(cuMemAddressReserve(&va_mc, sz, g, 0, 0));
  CK(cuMemMap(va_mc, sz, 0, mc, 0));
  CK(cuMemAddressReserve(&va_uc, sz, g, 0, 0));
  CK(cuMemMap(va_uc, sz, 0, mem, 0));
  CUmemAccessDesc ad = {};
  ad.location = ap.location;
  ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CK(cuMemSetAccess(va_mc, sz, &ad, 1));
  CK(cuMemSetAccess(va_uc, sz, &ad, 1));
  float* out;
  cudaMalloc(&out, 2 * 1024 * 4);
  k<<<1, 256>>>((float*)va_mc, (float*)va_uc, 1024, out);
  cudaError_t e = cudaDeviceSynchronize();
  printf("{\"kernel\": \"%s\"}\n", cudaGetErrorString(e));
  float h[2048];
  cudaMemcpy(h, out, sizeof h, cudaMemcpyDeviceToHost);
  int bad = 0;
  for (int i = 0; i < 1024; ++i) {
    float ex = (float)(1 + (i & 3)) + (float)(i & ~3);
    if (h[i] != ex || h[1024 + i] != ex) ++bad;
  }
  printf("{\"ld_reduce_and_unicast_mismatches\": %d, \"sample\": [%g, %g, %g]}\n", bad, h[5], h[1024 + 5], h[1023]);
  return 0;
}
