// Host-side cost of launch paths for a kernel with a ~224 B parameter block.
#include <chrono>
#include <cstdio>
#include <cuda.h>
#include <cuda_runtime.h>
struct Big { char b[224]; };
__global__ void k_big(Big a) { if (a.b[0] == 123 && threadIdx.x == 999) printf("x"); }
static double now_us() { return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count(); }
int main() {
    cudaStream_t st; cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
    Big a{}; const int N = 2000;
    k_big<<<148, 256, 0, st>>>(a); cudaStreamSynchronize(st);
    for (int mode = 0; mode < 4; mode++) {
        cudaGraphExec_t ge = nullptr;
        if (mode == 3) {
            cudaGraph_t g; cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
            k_big<<<148, 256, 0, st>>>(a); cudaStreamEndCapture(st, &g); cudaGraphInstantiate(&ge, g, 0);
        }
        CUfunction f; cudaGetFuncBySymbol((cudaFunction_t *)&f, (const void *)k_big);
        double tot = 0, idle = 0;
        for (int i = 0; i < N; i++) {
            double t0 = now_us();
            if (mode == 0) k_big<<<148, 256, 0, st>>>(a);
            else if (mode == 1) { cudaLaunchConfig_t c{}; c.gridDim = 148; c.blockDim = 256; c.stream = st; cudaLaunchKernelEx(&c, k_big, a); }
            else if (mode == 2) { void *args[] = {&a}; cuLaunchKernel(f, 148, 1, 1, 256, 1, 1, 0, (CUstream)st, args, nullptr); }
            else cudaGraphLaunch(ge, st);
            double t1 = now_us();
            tot += t1 - t0;
            if (i % 10 == 0) { cudaStreamSynchronize(st); }  // sometimes from idle
        }
        cudaStreamSynchronize(st);
        // idle-GPU launch: sync before every launch
        for (int i = 0; i < 200; i++) {
            cudaStreamSynchronize(st);
            double t0 = now_us();
            if (mode == 0) k_big<<<148, 256, 0, st>>>(a);
            else if (mode == 1) { cudaLaunchConfig_t c{}; c.gridDim = 148; c.blockDim = 256; c.stream = st; cudaLaunchKernelEx(&c, k_big, a); }
            else if (mode == 2) { void *args[] = {&a}; cuLaunchKernel(f, 148, 1, 1, 256, 1, 1, 0, (CUstream)st, args, nullptr); }
            else cudaGraphLaunch(ge, st);
            idle += now_us() - t0;
        }
        cudaStreamSynchronize(st);
        const char *nm[] = {"<<<>>>", "cudaLaunchKernelEx", "cuLaunchKernel", "cudaGraphLaunch"};
        printf("%-20s host %.2f us/launch (busy), %.2f us (idle GPU)\n", nm[mode], tot / N, idle / 200);
    }
    {   // graph node param update + launch (per-publish parameters)
        cudaGraph_t g; cudaGraphExec_t ge; cudaGraphNode_t node;
        cudaGraphCreate(&g, 0);
        cudaKernelNodeParams kp{}; void *args[] = {&a};
        kp.func = (void *)k_big; kp.gridDim = 148; kp.blockDim = 256; kp.kernelParams = args;
        cudaGraphAddKernelNode(&node, g, nullptr, 0, &kp);
        cudaGraphInstantiate(&ge, g, 0);
        double tot = 0;
        for (int i = 0; i < N; i++) {
            a.b[1] = (char)i;
            double t0 = now_us();
            cudaGraphExecKernelNodeSetParams(ge, node, &kp);
            cudaGraphLaunch(ge, st);
            tot += now_us() - t0;
            if (i % 10 == 0) cudaStreamSynchronize(st);
        }
        cudaStreamSynchronize(st);
        printf("%-20s host %.2f us/launch\n", "graph SetParams+Launch", tot / N);
    }
    // round trip: launch + sync on an idle GPU
    double rt = 0;
    for (int i = 0; i < 200; i++) { double t0 = now_us(); k_big<<<148, 256, 0, st>>>(a); cudaStreamSynchronize(st); rt += now_us() - t0; }
    printf("launch+sync round trip (idle): %.2f us\n", rt / 200);
    return 0;
}
