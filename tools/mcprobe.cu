#include <cstdio>
#include <cuda.h>
int main() {
    cuInit(0); CUdevice d; cuDeviceGet(&d, 0);
    int mc = -1, fab = -1, p2p = -1;
    cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, d);
    cuDeviceGetAttribute(&fab, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, d);
    cuDeviceGetAttribute(&p2p, CU_DEVICE_ATTRIBUTE_CAN_USE_64_BIT_STREAM_MEM_OPS, d);
    int ndev = 0; cuDeviceGetCount(&ndev);
    printf("devices=%d multicast_supported=%d fabric_handles=%d stream_mem_ops64=%d\n", ndev, mc, fab, p2p);
    if (mc == 1) {
        CUmulticastObjectProp prop{}; prop.numDevices = 1; prop.size = 2 << 20; prop.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
        size_t gran = 0; CUresult r = cuMulticastGetGranularity(&gran, &prop, CU_MULTICAST_GRANULARITY_RECOMMENDED);
        CUmemGenericAllocationHandle h; CUresult r2 = cuMulticastCreate(&h, &prop);
        printf("granularity=%zu (r=%d) create(1 device, fd)=%d\n", gran, r, r2);
        for (int ht : {0, (int)CU_MEM_HANDLE_TYPE_FABRIC}) {
            for (unsigned nd : {1u, 2u}) {
                CUmulticastObjectProp p2{}; p2.numDevices = nd; p2.size = 2 << 20; p2.handleTypes = ht;
                CUmemGenericAllocationHandle h2; CUresult r3 = cuMulticastCreate(&h2, &p2);
                CUresult r4 = CUDA_ERROR_UNKNOWN;
                if (r3 == CUDA_SUCCESS) r4 = cuMulticastAddDevice(h2, d);
                printf("create(numDevices=%u, handleTypes=%d)=%d addDevice=%d\n", nd, ht, r3, r4);
            }
        }
    }
    return 0;
}
