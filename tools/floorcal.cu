// Floor of "launch a grid, last block writes a host-mapped status word, host
// spins on it": what the SYNC fused publish pays besides moving bytes.
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>
static double now_us() { return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count(); }
__global__ void k_done(unsigned *done, volatile int *status, int token) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        if (atomicAdd(done, 1u) == gridDim.x - 1) { *done = 0; __threadfence(); *status = token; }
    }
}
int main() {
    cudaStream_t st; cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
    unsigned *done; cudaMalloc(&done, 4); cudaMemset(done, 0, 4);
    int *h; cudaHostAlloc(&h, 64, cudaHostAllocMapped); volatile int *hv = h; *hv = 0;
    int *d; cudaHostGetDevicePointer((void **)&d, h, 0);
    for (int grid : {1, 148, 282, 296}) {
        for (int mode = 0; mode < 2; mode++) {
            cudaGraph_t g; cudaGraphExec_t ge; cudaGraphNode_t node;
            int token = 1;
            void *args[] = {&done, &d, &token};
            cudaKernelNodeParams kp{}; kp.func = (void *)k_done; kp.gridDim = grid; kp.blockDim = 256; kp.kernelParams = args;
            cudaGraphCreate(&g, 0); cudaGraphAddKernelNode(&node, g, nullptr, 0, &kp); cudaGraphInstantiate(&ge, g, 0);
            double tot = 0; int n = 0;
            for (int i = 1; i <= 300; i++) {
                token = i;
                cudaStreamSynchronize(st);
                double t0 = now_us();
                if (mode == 0) { cudaGraphExecKernelNodeSetParams(ge, node, &kp); cudaGraphLaunch(ge, st); }
                else k_done<<<grid, 256, 0, st>>>(done, d, i);
                while (*hv != i) {}
                double t1 = now_us();
                if (i > 20) { tot += t1 - t0; n++; }
            }
            printf("grid %3d %-8s launch -> host sees status: %.2f us\n", grid, mode ? "<<<>>>" : "graph", tot / n);
        }
    }
    return 0;
}
