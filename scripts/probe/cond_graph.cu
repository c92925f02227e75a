#include <cuda_runtime.h>
#include <cstdio>
__global__ void k_cond(cudaGraphConditionalHandle h, int *st) {
  cudaGraphSetConditional(h, *st != 0 ? 1u : 0u);
}
__global__ void k_body(int *st, int *cnt) { if (++*cnt >= 5) *st = 0; }
__global__ void k_pdl(int *cnt) { asm volatile("griddepcontrol.wait;" ::: "memory"); cnt[1] += 1; }
extern "C" int run() {
  cudaStream_t s; cudaStreamCreate(&s);
  int *d; cudaMalloc(&d, 16); cudaMemset(d, 0, 16); int one = 1; cudaMemcpy(d, &one, 4, cudaMemcpyHostToDevice);
  cudaGraph_t g; cudaGraphCreate(&g, 0);
  cudaGraphConditionalHandle h;
  cudaError_t e = cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault);
  if (e) { printf("handle %s\n", cudaGetErrorString(e)); return 1; }
  cudaGraphNodeParams cp = {};
  cp.type = cudaGraphNodeTypeConditional;
  cp.conditional.handle = h;
  cp.conditional.type = cudaGraphCondTypeWhile;
  cp.conditional.size = 1;
  cudaGraphNode_t node;
  e = cudaGraphAddNode(&node, g, nullptr, 0, &cp);
  if (e) { printf("addnode %s\n", cudaGetErrorString(e)); return 1; }
  cudaGraph_t body = cp.conditional.phGraph_out[0];
  e = cudaStreamBeginCaptureToGraph(s, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed);
  if (e) { printf("capture %s\n", cudaGetErrorString(e)); return 1; }
  k_body<<<1,1,0,s>>>(d, d+1);
  {
    cudaLaunchConfig_t cfg = {}; cfg.gridDim = dim3(1); cfg.blockDim = dim3(1); cfg.stream = s;
    cudaLaunchAttribute at[1]; at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1; cfg.attrs = at; cfg.numAttrs = 1;
    e = cudaLaunchKernelEx(&cfg, k_pdl, d + 1);
    if (e) { printf("pdl %s\n", cudaGetErrorString(e)); return 1; }
  }
  k_cond<<<1,1,0,s>>>(h, d);
  e = cudaStreamEndCapture(s, &body);
  if (e) { printf("endcap %s\n", cudaGetErrorString(e)); return 1; }
  cudaGraphExec_t x; e = cudaGraphInstantiate(&x, g, 0);
  if (e) { printf("inst %s\n", cudaGetErrorString(e)); return 1; }
  cudaGraphLaunch(x, s); cudaStreamSynchronize(s);
  int hv[3]; cudaMemcpy(hv, d, 12, cudaMemcpyDeviceToHost);
  printf("st=%d cnt=%d pdl=%d err=%s\n", hv[0], hv[1], hv[2], cudaGetErrorString(cudaGetLastError()));
  return 0;
}
int main() { return run(); }
