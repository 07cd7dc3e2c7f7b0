// Probe of NVSwitch multicast object creation on this box (reading R23 hardware form):
// cuMulticastCreate over a grid of (numDevices, handle type, size), then AddDevice / BindMem
// for the visible devices. Prints one line per attempt with the CUresult.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdio.h>
int main() {
  cudaFree(0);
  int ndev = 0;
  cudaGetDeviceCount(&ndev);
  int sup = 0;
  cuDeviceGetAttribute(&sup, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, 0);
  int drv = 0;
  cuDriverGetVersion(&drv);
  printf("devices %d multicast_supported %d driver %d\n", ndev, sup, drv);
  unsigned long long hts[3] = {0, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, CU_MEM_HANDLE_TYPE_FABRIC};
  for (int nd = 1; nd <= 2; nd++)
    for (int h = 0; h < 3; h++)
      for (size_t sz : {(size_t)2 << 20, (size_t)512 << 20}) {
        CUmulticastObjectProp p = {};
        p.numDevices = nd;
        p.size = sz;
        p.handleTypes = hts[h];
        size_t g = 0;
        CUresult eg = cuMulticastGetGranularity(&g, &p, CU_MULTICAST_GRANULARITY_RECOMMENDED);
        CUmemGenericAllocationHandle mc = 0;
        CUresult ec = cuMulticastCreate(&mc, &p);
        CUresult ea = CUDA_ERROR_UNKNOWN, eb = CUDA_ERROR_UNKNOWN;
        if (ec == CUDA_SUCCESS) {
          ea = cuMulticastAddDevice(mc, 0);
          CUmemAllocationProp ap = {};
          ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
          ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
          ap.location.id = 0;
          ap.requestedHandleTypes = (CUmemAllocationHandleType)hts[h];
          CUmemGenericAllocationHandle phys;
          if (cuMemCreate(&phys, sz, &ap, 0) == CUDA_SUCCESS) {
            eb = cuMulticastBindMem(mc, 0, phys, 0, sz, 0);
            cuMemRelease(phys);
          }
          cuMemRelease(mc);
        }
        printf("numDevices %d handleType %llu size %zu: granularity %d (%zu) create %d addDevice %d bind %d\n", nd,
               hts[h], sz, (int)eg, g, (int)ec, (int)ea, (int)eb);
      }
  return 0;
}
