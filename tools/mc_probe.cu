// mc_probe.cu — does this B200 support NVLS multicast objects (cuMulticast*) and
// multimem.st through them? One device: create a multicast object, bind a
// physical allocation, map the multicast address, store through it with
// multimem.st from a kernel, read the bound memory back.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tools/mc_probe tools/mc_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <vector>

#define CU(x)                                                                  \
  do {                                                                         \
    CUresult r_ = (x);                                                         \
    if (r_ != CUDA_SUCCESS) {                                                  \
      const char *s_ = nullptr;                                                \
      cuGetErrorString(r_, &s_);                                               \
      printf("%s -> %d %s\n", #x, (int)r_, s_ ? s_ : "?");                     \
      return 1;                                                                \
    }                                                                          \
  } while (0)

__global__ void k_mc_store(float *mc, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const float v = (float)i * 0.5f;
    asm volatile("multimem.st.global.f32 [%0], %1;" ::"l"(mc + i), "f"(v) : "memory");
  }
}

int main() {
  CU(cuInit(0));
  CUdevice dev;
  CU(cuDeviceGet(&dev, 0));
  int mc = 0, fabric = 0;
  cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev);
  cuDeviceGetAttribute(&fabric, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, dev);
  printf("multicast supported: %d, fabric handles: %d\n", mc, fabric);
  cudaSetDevice(0);
  cudaFree(nullptr);
  if (!mc) return 0;
  const int n = 1 << 20;
  const size_t bytes = sizeof(float) * n;
  CUmulticastObjectProp mp = {};
  mp.numDevices = 1;
  size_t gran = 0;
  mp.size = bytes;
  CUmemGenericAllocationHandle mch;
  size_t size = 0;
  bool made = false;
  for (CUmemAllocationHandleType ht : {CU_MEM_HANDLE_TYPE_FABRIC, CU_MEM_HANDLE_TYPE_NONE,
                                       CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR}) {
    mp.handleTypes = ht;
    mp.size = bytes;
    CUresult g = cuMulticastGetGranularity(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED);
    if (g != CUDA_SUCCESS) { printf("granularity (handle type %d) -> %d\n", (int)ht, (int)g); continue; }
    size = (bytes + gran - 1) / gran * gran;
    mp.size = size;
    CUresult r = cuMulticastCreate(&mch, &mp);
    printf("cuMulticastCreate(handle type %d, size %zu, gran %zu) -> %d\n", (int)ht, size, gran, (int)r);
    if (r == CUDA_SUCCESS) { made = true; break; }
  }
  if (!made) return 0;
  CU(cuMulticastAddDevice(mch, dev));
  CUmemAllocationProp ap = {};
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = 0;
  ap.requestedHandleTypes = (CUmemAllocationHandleType)mp.handleTypes;
  CUmemGenericAllocationHandle ph;
  CU(cuMemCreate(&ph, size, &ap, 0));
  CU(cuMulticastBindMem(mch, 0, ph, 0, size, 0));
  CUdeviceptr uc = 0, mcp = 0;
  CU(cuMemAddressReserve(&uc, size, gran, 0, 0));
  CU(cuMemMap(uc, size, 0, ph, 0));
  CU(cuMemAddressReserve(&mcp, size, gran, 0, 0));
  CU(cuMemMap(mcp, size, 0, mch, 0));
  CUmemAccessDesc ad = {};
  ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ad.location.id = 0;
  ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CU(cuMemSetAccess(uc, size, &ad, 1));
  CU(cuMemSetAccess(mcp, size, &ad, 1));
  k_mc_store<<<148, 256>>>((float *)mcp, n);
  cudaError_t e = cudaDeviceSynchronize();
  printf("multimem.st kernel: %s\n", cudaGetErrorString(e));
  std::vector<float> h(n);
  cudaMemcpy(h.data(), (void *)uc, bytes, cudaMemcpyDeviceToHost);
  int bad = 0;
  for (int i = 0; i < n; i++) bad += h[i] != (float)i * 0.5f;
  printf("bound memory after multimem.st: %d of %d wrong\n", bad, n);
  return 0;
}
