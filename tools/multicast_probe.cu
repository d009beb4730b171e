// multicast_probe.cu — can this box run NVLS (multimem) collectives with one
// visible GPU? Creates a 1-device multicast object, binds a buffer, maps the
// multicast address and runs multimem.st / multimem.red.add /
// multimem.ld_reduce.add on it. Prints each step's result.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tools/multicast_probe tools/multicast_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstring>

#define CK(x)                                                                  \
  do {                                                                         \
    CUresult r_ = (x);                                                         \
    if (r_ != CUDA_SUCCESS) {                                                  \
      const char* s_ = nullptr;                                                \
      cuGetErrorString(r_, &s_);                                               \
      printf("FAIL %s: %d %s\n", #x, int(r_), s_ ? s_ : "?");                 \
      return 1;                                                                \
    }                                                                          \
  } while (0)

__global__ void mm_kernel(float* mc, float* uc, float* out, int n) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  // multimem.st: write 1.0 to every device's copy
  asm volatile("multimem.st.global.f32 [%0], %1;" ::"l"(mc + i), "f"(1.0f) : "memory");
  asm volatile("fence.proxy.alias;" ::: "memory");
  // multimem.red.add: add 2.0 to every copy
  asm volatile("multimem.red.global.add.f32 [%0], %1;" ::"l"(mc + i), "f"(2.0f) : "memory");
  asm volatile("fence.proxy.alias;" ::: "memory");
  __threadfence_system();
  float v;
  asm volatile("multimem.ld_reduce.global.add.f32 %0, [%1];" : "=f"(v) : "l"(mc + i) : "memory");
  out[i] = v;
  out[n + i] = uc[i];
}

int main() {
  CK(cuInit(0));
  CUdevice dev;
  CK(cuDeviceGet(&dev, 0));
  int mc = -1, fab = -1, vmm = -1;
  cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev);
  cuDeviceGetAttribute(&vmm, CU_DEVICE_ATTRIBUTE_VIRTUAL_MEMORY_MANAGEMENT_SUPPORTED, dev);
#ifdef CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED
  cuDeviceGetAttribute(&fab, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, dev);
#endif
  printf("multicast_supported=%d vmm=%d fabric_handles=%d\n", mc, vmm, fab);
  CUcontext ctx;
  CK(cuDevicePrimaryCtxRetain(&ctx, dev));
  CK(cuCtxSetCurrent(ctx));
  if (mc != 1) {
    printf("RESULT: multicast unsupported on this device\n");
    return 0;
  }
  const int n = 1 << 16;
  CUmulticastObjectProp mp;
  CUmemGenericAllocationHandle mch;
  const CUmemAllocationHandleType types[3] = {CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, CU_MEM_HANDLE_TYPE_NONE,
                                              CU_MEM_HANDLE_TYPE_FABRIC};
  int ok = -1;
  for (int ti = 0; ti < 3 && ok < 0; ++ti) {
    for (int nd = 1; nd <= 2 && ok < 0; ++nd) {
      std::memset(&mp, 0, sizeof(mp));
      mp.numDevices = nd;
      mp.handleTypes = types[ti];
      size_t gran = 0;
      mp.size = n * sizeof(float);
      CUresult r = cuMulticastGetGranularity(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED);
      if (r == CUDA_SUCCESS) mp.size = ((n * sizeof(float) + gran - 1) / gran) * gran;
      r = cuMulticastCreate(&mch, &mp);
      const char* es = nullptr;
      cuGetErrorString(r, &es);
      printf("cuMulticastCreate(handleType=%d, numDevices=%d, size=%zu): %d %s\n", int(types[ti]), nd, mp.size, int(r),
             es ? es : "?");
      if (r == CUDA_SUCCESS) ok = ti;
    }
  }
  if (ok < 0) {
    printf("RESULT: cuMulticastCreate fails for every handle type (no NVSwitch fabric reachable)\n");
    return 0;
  }
  CK(cuMulticastAddDevice(mch, dev));
  CUmemAllocationProp ap;
  std::memset(&ap, 0, sizeof(ap));
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = 0;
  ap.requestedHandleTypes = CUmemAllocationHandleType(mp.handleTypes);
  size_t ag = 0;
  CK(cuMemGetAllocationGranularity(&ag, &ap, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
  const size_t bytes = ((mp.size + ag - 1) / ag) * ag;
  CUmemGenericAllocationHandle uh;
  CK(cuMemCreate(&uh, bytes, &ap, 0));
  CK(cuMulticastBindMem(mch, 0, uh, 0, bytes, 0));
  CUdeviceptr ua = 0, ma = 0;
  CK(cuMemAddressReserve(&ua, bytes, 0, 0, 0));
  CK(cuMemMap(ua, bytes, 0, uh, 0));
  CUmemAccessDesc ad;
  ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ad.location.id = 0;
  ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CK(cuMemSetAccess(ua, bytes, &ad, 1));
  CK(cuMemAddressReserve(&ma, mp.size, 0, 0, 0));
  CK(cuMemMap(ma, mp.size, 0, mch, 0));
  CK(cuMemSetAccess(ma, mp.size, &ad, 1));
  float* out = nullptr;
  cudaMalloc(&out, 2 * n * sizeof(float));
  mm_kernel<<<n / 256, 256>>>(reinterpret_cast<float*>(ma), reinterpret_cast<float*>(ua), out, n);
  cudaError_t e = cudaDeviceSynchronize();
  printf("kernel: %s\n", cudaGetErrorString(e));
  if (e != cudaSuccess) return 1;
  float h[4];
  cudaMemcpy(h, out, sizeof(float), cudaMemcpyDeviceToHost);
  cudaMemcpy(h + 1, out + n, sizeof(float), cudaMemcpyDeviceToHost);
  printf("ld_reduce=%g unicast=%g (want 3, 3)\n", h[0], h[1]);
  printf("RESULT: multicast %s\n", (h[0] == 3.0f && h[1] == 3.0f) ? "works" : "wrong values");
  return 0;
}
