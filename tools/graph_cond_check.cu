// Minimal reproducer for compute-sanitizer and device-side graph conditionals:
// a while-node whose body kernel counts to N and then ends the loop with
// cudaGraphSetConditional (the pattern of the PCG loop graph, capi.cpp).
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tools/graph_cond_check tools/graph_cond_check.cu
//   compute-sanitizer --tool memcheck tools/graph_cond_check
#include <cstdio>
#include <cuda_runtime.h>

__global__ void body(int* counter, int n, cudaGraphConditionalHandle h) {
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        int c = ++*counter;
        if (c >= n) cudaGraphSetConditional(h, 0);
    }
}

// second kernel of the body (the PCG body is A, B, A, B): also ends the loop
// once the count is reached, from the LAST block
__global__ void body2(const int* counter, int n, cudaGraphConditionalHandle h) {
    if (threadIdx.x == 0 && blockIdx.x == gridDim.x - 1 && *counter >= n) cudaGraphSetConditional(h, 0);
}

int main() {
    int* d;
    cudaMalloc(&d, sizeof(int));
    cudaMemset(d, 0, sizeof(int));
    cudaGraph_t g;
    cudaGraphCreate(&g, 0);
    cudaGraphConditionalHandle h;
    cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault);
    cudaGraphNodeParams p = {};
    p.type = cudaGraphNodeTypeConditional;
    p.conditional.handle = h;
    p.conditional.type = cudaGraphCondTypeWhile;
    p.conditional.size = 1;
    cudaGraphNode_t node;
    cudaGraphAddNode(&node, g, nullptr, 0, &p);
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaStreamBeginCaptureToGraph(s, p.conditional.phGraph_out[0], nullptr, nullptr, 0,
                                  cudaStreamCaptureModeThreadLocal);
    body<<<4, 64, 0, s>>>(d, 10, h);
    body2<<<300, 64, 0, s>>>(d, 10, h);
    body<<<4, 64, 0, s>>>(d, 10, h);
    body2<<<300, 64, 0, s>>>(d, 10, h);
    cudaGraph_t out;
    cudaStreamEndCapture(s, &out);
    cudaGraphExec_t ge;
    cudaError_t e = cudaGraphInstantiate(&ge, g, 0);
    // as in mas_pcg_solve: ordinary launches of the same kernels (handle 0,
    // i.e. outside the graph) on the stream right before the graph launch
    body2<<<300, 64, 0, s>>>(d, 1 << 30, 0);
    if (e == cudaSuccess) e = cudaGraphLaunch(ge, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    int c = -1;
    cudaMemcpy(&c, d, sizeof(int), cudaMemcpyDeviceToHost);
    printf("status %s, iterations %d (expect 10)\n", cudaGetErrorString(e), c);
    return e == cudaSuccess && c == 10 ? 0 : 1;
}
