#include <cstdio>
#include <cuda_runtime.h>
__global__ void k_begin(int *cnt, cudaGraphConditionalHandle h) { cudaGraphSetConditional(h, *cnt > 0); }
__global__ void k_body(int *cnt, int *acc, cudaGraphConditionalHandle h) { *acc += *cnt; (*cnt)--; cudaGraphSetConditional(h, *cnt > 0); }
int main() {
  int *d; cudaMalloc(&d, 8);
  cudaGraph_t g; cudaGraphCreate(&g, 0);
  cudaGraphConditionalHandle h; cudaGraphConditionalHandleCreate(&h, g, 0, 0);
  cudaStream_t s; cudaStreamCreate(&s);
  // node 1: begin kernel via capture-to-graph
  cudaStreamBeginCaptureToGraph(s, g, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed);
  k_begin<<<1,1,0,s>>>(d, h);
  const cudaGraphNode_t *deps; size_t nd; cudaStreamCaptureStatus cs; cudaGraph_t cg;
  cudaStreamGetCaptureInfo(s, &cs, nullptr, &cg, &deps, &nd);
  cudaGraphNodeParams cp = {};
  cp.type = cudaGraphNodeTypeConditional;
  cp.conditional.handle = h; cp.conditional.type = cudaGraphCondTypeWhile; cp.conditional.size = 1;
  cudaGraphNode_t cn;
  cudaError_t e = cudaGraphAddNode(&cn, cg, deps, nd, &cp);
  printf("add %s\n", cudaGetErrorString(e));
  cudaStreamUpdateCaptureDependencies(s, &cn, 1, cudaStreamSetCaptureDependencies);
  cudaGraph_t body = cp.conditional.phGraph_out[0];
  cudaGraph_t dummy; e = cudaStreamEndCapture(s, &dummy); printf("end %s\n", cudaGetErrorString(e));
  cudaStreamBeginCaptureToGraph(s, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed);
  k_body<<<1,1,0,s>>>(d, d+1, h);
  e = cudaStreamEndCapture(s, &dummy); printf("end2 %s\n", cudaGetErrorString(e));
  cudaGraphExec_t x; e = cudaGraphInstantiate(&x, g, 0); printf("inst %s\n", cudaGetErrorString(e));
  for (int r = 0; r < 3; r++) {
    int v[2] = {5 + r, 0}; cudaMemcpyAsync(d, v, 8, cudaMemcpyHostToDevice, s);
    cudaGraphLaunch(x, s); cudaMemcpyAsync(v, d, 8, cudaMemcpyDeviceToHost, s); cudaStreamSynchronize(s);
    printf("cnt %d acc %d (expect %d)\n", v[0], v[1], (5+r)*(6+r)/2);
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
