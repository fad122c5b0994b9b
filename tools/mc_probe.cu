// Probe: can this GPU create an NVLink SHARP multicast object (cuMulticastCreate) and run
// multimem.st / multimem.red on it?  Prints the capability attributes and a self-check.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/mc_probe tools/mc_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#define CKD(x) do { CUresult r_ = (x); if (r_ != CUDA_SUCCESS) { const char* s_; cuGetErrorString(r_, &s_); \
    printf("FAIL %s -> %d %s\n", #x, (int)r_, s_); return 1; } } while (0)

__global__ void k_mc(unsigned* mc32, unsigned long long* mc64, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) {
        asm volatile("multimem.st.relaxed.sys.global.b32 [%0], %1;" :: "l"(mc32 + i), "r"((unsigned)(i * 3 + 1)) : "memory");
        asm volatile("multimem.red.relaxed.sys.global.add.u64 [%0], %1;" :: "l"(mc64 + (i & 15)), "l"(1ull) : "memory");
    }
}

int main() {
    CKD(cuInit(0));
    CUdevice d;
    CKD(cuDeviceGet(&d, 0));
    cudaSetDevice(0);
    cudaFree(0);
    int mc = 0, fab = 0, posix = 0, vmm = 0;
    cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, d);
    cuDeviceGetAttribute(&fab, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, d);
    cuDeviceGetAttribute(&posix, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR_SUPPORTED, d);
    cuDeviceGetAttribute(&vmm, CU_DEVICE_ATTRIBUTE_VIRTUAL_MEMORY_MANAGEMENT_SUPPORTED, d);
    int ndev = 0;
    cudaGetDeviceCount(&ndev);
    printf("devices %d multicast %d fabric_handle %d posix_fd %d vmm %d\n", ndev, mc, fab, posix, vmm);
    if (!mc) { printf("NO MULTICAST\n"); return 0; }
    CUmulticastObjectProp p = {};
    p.numDevices = 1;
    p.size = 2 << 20;
    size_t gran = 0;
    CUmemGenericAllocationHandle mch, mh;
    // which handle types does cuMulticastCreate accept here?
    const unsigned long long types[3] = {0ull, (unsigned long long)CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR,
                                         (unsigned long long)CU_MEM_HANDLE_TYPE_FABRIC};
    int ok_type = -1;
    for (int t = 0; t < 3; ++t) {
        for (int nd = 1; nd <= 2; ++nd) {
            p.handleTypes = types[t];
            p.numDevices = nd;
            CUresult rg = cuMulticastGetGranularity(&gran, &p, CU_MULTICAST_GRANULARITY_RECOMMENDED);
            p.size = gran ? ((2 << 20) + gran - 1) / gran * gran : (2 << 20);
            CUresult rc = cuMulticastCreate(&mch, &p);
            const char* es = nullptr;
            cuGetErrorString(rc, &es);
            printf("handleTypes %llu numDevices %d: granularity rc %d (%zu), create rc %d %s\n", types[t], nd, (int)rg,
                   gran, (int)rc, es);
            if (rc == CUDA_SUCCESS) {
                if (nd == 1 && ok_type < 0) ok_type = t;
                else cuMemRelease(mch);
                if (nd == 1) goto made;
            }
        }
    }
    printf("NO MULTICAST OBJECT\n");
    return 0;
made:
    size_t size = p.size;
    CKD(cuMulticastAddDevice(mch, d));
    CUmemAllocationProp ap = {};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = 0;
    ap.requestedHandleTypes = (CUmemAllocationHandleType)types[ok_type];
    size_t mg = 0;
    CKD(cuMemGetAllocationGranularity(&mg, &ap, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
    CKD(cuMemCreate(&mh, size, &ap, 0));
    CKD(cuMulticastBindMem(mch, 0, mh, 0, size, 0));
    CUdeviceptr uc, mcp;
    CKD(cuMemAddressReserve(&uc, size, gran, 0, 0));
    CKD(cuMemMap(uc, size, 0, mh, 0));
    CUmemAccessDesc ad = {};
    ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ad.location.id = 0;
    ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CKD(cuMemSetAccess(uc, size, &ad, 1));
    CKD(cuMemAddressReserve(&mcp, size, gran, 0, 0));
    CKD(cuMemMap(mcp, size, 0, mch, 0));
    CKD(cuMemSetAccess(mcp, size, &ad, 1));
    cudaMemset((void*)uc, 0, size);
    const int n = 4096;
    unsigned* mc32 = (unsigned*)mcp;
    unsigned long long* mc64 = (unsigned long long*)(mcp + 65536);
    k_mc<<<n / 256, 256>>>(mc32, mc64, n);
    cudaError_t e = cudaDeviceSynchronize();
    printf("kernel: %s\n", cudaGetErrorString(e));
    unsigned h32[n];
    unsigned long long h64[16];
    cudaMemcpy(h32, (void*)uc, sizeof(h32), cudaMemcpyDeviceToHost);
    cudaMemcpy(h64, (void*)(uc + 65536), sizeof(h64), cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int i = 0; i < n; ++i) bad += h32[i] != (unsigned)(i * 3 + 1);
    for (int i = 0; i < 16; ++i) bad += h64[i] != (unsigned long long)(n / 16);
    printf("multimem check: %s (%d bad)\n", bad ? "FAIL" : "OK", bad);
    return 0;
}
