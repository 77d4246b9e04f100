// Prints the shared-window offset of dynamic shared memory for a kernel with
// no static shared memory (the scan's table addressing assumes it; standalone).
#include <cstdio>
#include <cstdint>
__global__ void k(uint32_t* out) {
    extern __shared__ uint8_t smem[];
    out[0] = (uint32_t)__cvta_generic_to_shared(smem);
}
int main() {
    uint32_t* d; uint32_t h = 0;
    cudaMalloc(&d, 4);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
    k<<<1, 32, 65536>>>(d);
    cudaMemcpy(&h, d, 4, cudaMemcpyDeviceToHost);
    int r = 0; cudaDeviceGetAttribute(&r, cudaDevAttrReservedSharedMemoryPerBlock, 0);
    printf("dynamic smem window offset %u, reserved per block %d, err %s\n", h, r, cudaGetErrorString(cudaGetLastError()));
}
