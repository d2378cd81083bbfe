// Second reproducer for compute-sanitizer racecheck / synccheck on the PCG
// loop graph's structure (capi.cpp loop_graph): a top-level graph holding a
// chain of kernel nodes (iteration 1) followed by a conditional WHILE node
// whose body kernels use an opt-in dynamic shared-memory size above 48 KB
// (as k_stencil and k_aniso do), barriers, and end the loop from a device-side
// cudaGraphSetConditional.  Argument: dynamic smem bytes (default 100 KB).
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tools/graph_cond_check2 tools/graph_cond_check2.cu
//   compute-sanitizer --tool racecheck tools/graph_cond_check2 [bytes]
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

__global__ void body(int* counter, int n, cudaGraphConditionalHandle h, int words) {
    extern __shared__ double sm[];
    for (int t = threadIdx.x; t < words; t += blockDim.x) sm[t] = (double)t;
    __syncthreads();
    double s = 0.0;
    for (int t = threadIdx.x; t < words; t += blockDim.x) s += sm[words - 1 - t];
    __syncthreads();
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        int c = ++*counter;
        if (c >= n && h) cudaGraphSetConditional(h, 0);
        if (s == -1.0) *counter = 0;  // keep s live
    }
}

int main(int argc, char** argv) {
    const int bytes = argc > 1 ? atoi(argv[1]) : 100 * 1024;
    const int words = bytes / 8;
    cudaError_t e = cudaFuncSetAttribute(body, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e != cudaSuccess) { printf("attr: %s\n", cudaGetErrorString(e)); return 1; }
    int* d;
    cudaMalloc(&d, sizeof(int));
    cudaMemset(d, 0, sizeof(int));
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaGraph_t g;
    cudaGraphCreate(&g, 0);
    // iteration 1: captured into the top-level graph
    cudaStreamBeginCaptureToGraph(s, g, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal);
    body<<<8, 256, bytes, s>>>(d, 1 << 30, 0, words);
    body<<<8, 256, bytes, s>>>(d, 1 << 30, 0, words);
    cudaGraph_t tmp = g;
    cudaStreamEndCapture(s, &tmp);
    size_t n = 0;
    cudaGraphGetNodes(g, nullptr, &n);
    cudaGraphNode_t nodes[8];
    cudaGraphGetNodes(g, nodes, &n);
    cudaGraphNode_t leaf = nullptr;
    for (size_t i = 0; i < n; i++) {
        size_t nd = 0;
        cudaGraphNodeGetDependentNodes(nodes[i], nullptr, &nd);
        if (nd == 0) leaf = nodes[i];
    }
    cudaGraphConditionalHandle h;
    cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault);
    cudaGraphNodeParams p = {};
    p.type = cudaGraphNodeTypeConditional;
    p.conditional.handle = h;
    p.conditional.type = cudaGraphCondTypeWhile;
    p.conditional.size = 1;
    cudaGraphNode_t node;
    e = cudaGraphAddNode(&node, g, &leaf, 1, &p);
    if (e != cudaSuccess) { printf("add: %s\n", cudaGetErrorString(e)); return 1; }
    cudaStreamBeginCaptureToGraph(s, p.conditional.phGraph_out[0], nullptr, nullptr, 0,
                                  cudaStreamCaptureModeThreadLocal);
    body<<<8, 256, bytes, s>>>(d, 12, h, words);
    body<<<8, 256, bytes, s>>>(d, 12, h, words);
    cudaGraph_t out;
    cudaStreamEndCapture(s, &out);
    cudaGraphExec_t ge;
    e = cudaGraphInstantiate(&ge, g, 0);
    if (e == cudaSuccess) e = cudaGraphLaunch(ge, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    int c = -1;
    cudaMemcpy(&c, d, sizeof(int), cudaMemcpyDeviceToHost);
    printf("smem %d B: status %s, count %d (expect 12 or 13)\n", bytes, cudaGetErrorString(e), c);
    return e == cudaSuccess && (c == 12 || c == 13) ? 0 : 1;
}
