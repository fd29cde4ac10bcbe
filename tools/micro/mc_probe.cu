// Probe: can this B200 build a one-member multicast object (NVLS) and run
// multimem.ld_reduce.min.s64 on it?  nvcc -gencode arch=compute_100a,code=sm_100a -o mc_probe mc_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#define CK(x) do { CUresult r = (x); if (r != CUDA_SUCCESS) { const char* s; cuGetErrorString(r, &s); \
    printf("FAIL %s: %s\n", #x, s); return 1; } } while (0)

__global__ void k_reduce(const long long* mc, long long* out, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) {
        long long v;
        asm volatile("multimem.ld_reduce.relaxed.sys.global.min.s64 %0, [%1];" : "=l"(v) : "l"(mc + i) : "memory");
        out[i] = v;
    }
}

int main() {
    CK(cuInit(0));
    CUdevice dev;
    CK(cuDeviceGet(&dev, 0));
    CUcontext ctx;
    CK(cuDevicePrimaryCtxRetain(&ctx, dev));
    CK(cuCtxSetCurrent(ctx));
    int mc = 0;
    CK(cuDeviceGetAttribute(&mc, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
    printf("multicast supported: %d\n", mc);
    if (!mc) return 0;
    const size_t n = 1 << 20, bytes = n * 8;
    CUmulticastObjectProp prop = {};
    prop.numDevices = 1;
    prop.size = bytes;
    prop.handleTypes = CU_MEM_HANDLE_TYPE_NONE;
    size_t gran = 0, mgran = 0;
    CK(cuMulticastGetGranularity(&mgran, &prop, CU_MULTICAST_GRANULARITY_MINIMUM));
    CK(cuMulticastGetGranularity(&gran, &prop, CU_MULTICAST_GRANULARITY_RECOMMENDED));
    printf("granularity min %zu rec %zu\n", mgran, gran);
    gran = mgran;
    prop.size = (bytes + gran - 1) / gran * gran;
    printf("granularity %zu size %zu\n", gran, prop.size);
    CUmemGenericAllocationHandle mch;
    CK(cuMulticastCreate(&mch, &prop));
    CK(cuMulticastAddDevice(mch, dev));
    CUmemAllocationProp ap = {};
    ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ap.location.id = 0;
    ap.requestedHandleTypes = CU_MEM_HANDLE_TYPE_NONE;
    CUmemGenericAllocationHandle ph;
    CK(cuMemCreate(&ph, prop.size, &ap, 0));
    CK(cuMulticastBindMem(mch, 0, ph, 0, prop.size, 0));
    CUdeviceptr uc, mcp;
    CK(cuMemAddressReserve(&uc, prop.size, gran, 0, 0));
    CK(cuMemMap(uc, prop.size, 0, ph, 0));
    CK(cuMemAddressReserve(&mcp, prop.size, gran, 0, 0));
    CK(cuMemMap(mcp, prop.size, 0, mch, 0));
    CUmemAccessDesc ad = {};
    ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    ad.location.id = 0;
    ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    CK(cuMemSetAccess(uc, prop.size, &ad, 1));
    CK(cuMemSetAccess(mcp, prop.size, &ad, 1));
    long long* h = new long long[n];
    for (size_t i = 0; i < n; ++i) h[i] = (long long)(i * 2654435761ull % 1000003) - 500000;
    cudaMemcpy((void*)uc, h, bytes, cudaMemcpyHostToDevice);
    long long* out;
    cudaMalloc(&out, bytes);
    k_reduce<<<(n + 255) / 256, 256>>>((const long long*)mcp, out, (int)n);
    cudaError_t e = cudaDeviceSynchronize();
    printf("kernel: %s\n", cudaGetErrorString(e));
    long long* o = new long long[n];
    cudaMemcpy(o, out, bytes, cudaMemcpyDeviceToHost);
    size_t bad = 0;
    for (size_t i = 0; i < n; ++i) bad += o[i] != h[i];
    printf("multimem.ld_reduce.min.s64 over a 1-member group: %zu mismatches of %zu\n", bad, n);
    return 0;
}
