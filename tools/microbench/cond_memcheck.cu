// Minimal repro for the open sanitizer item (DESIGN.md §8 "Sanitizers"):
// does compute-sanitizer memcheck fail a CUDA-graph conditional WHILE node
// whose body kernel sets the condition from device code, with none of the
// shard-pass code involved?
//   nvcc -gencode arch=compute_100a,code=sm_100a -o cond_memcheck cond_memcheck.cu -lcudadevrt -rdc=true
//   ./cond_memcheck [runs] [pad]; compute-sanitizer --tool memcheck ./cond_memcheck [runs] [pad]
// `pad` > 0 passes a large by-value parameter struct (like the shard pass's KParams).
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

struct Ctl { unsigned iter, max_iters; };
struct Big {
  Ctl* ctl;
  unsigned long long pad[48];
  cudaGraphConditionalHandle h;
};

__global__ void body_small(Ctl* ctl, cudaGraphConditionalHandle h) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    const unsigned n = ++ctl->iter;
    cudaGraphSetConditional(h, n < ctl->max_iters ? 1u : 0u);
  }
}

__global__ void body_big(Big p) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    const unsigned n = ++p.ctl->iter;
    cudaGraphSetConditional(p.h, n < p.ctl->max_iters ? 1u : 0u);
  }
}

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  std::printf("%s:%d %s -> %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); return 1; } } while (0)

int main(int argc, char** argv) {
  const int runs = argc > 1 ? std::atoi(argv[1]) : 5;
  const int big = argc > 2 ? std::atoi(argv[2]) : 0;
  Ctl* ctl;
  CK(cudaMalloc(&ctl, sizeof(Ctl)));
  cudaStream_t s;
  CK(cudaStreamCreate(&s));
  cudaGraph_t graph;
  CK(cudaGraphCreate(&graph, 0));
  cudaGraphConditionalHandle h;
  CK(cudaGraphConditionalHandleCreate(&h, graph, 1, cudaGraphCondAssignDefault));
  cudaGraphNodeParams cp = {};
  cp.type = cudaGraphNodeTypeConditional;
  cp.conditional.handle = h;
  cp.conditional.type = cudaGraphCondTypeWhile;
  cp.conditional.size = 1;
  cudaGraphNode_t cn;
  CK(cudaGraphAddNode(&cn, graph, nullptr, 0, &cp));
  cudaGraph_t bodyg = cp.conditional.phGraph_out[0];
  Big bp = {};
  bp.ctl = ctl;
  bp.h = h;
  void* args_small[] = {&ctl, &h};
  void* args_big[] = {&bp};
  cudaKernelNodeParams kp = {};
  kp.func = big ? (void*)body_big : (void*)body_small;
  kp.gridDim = dim3(148);
  kp.blockDim = dim3(256);
  kp.kernelParams = big ? args_big : args_small;
  cudaGraphNode_t kn;
  CK(cudaGraphAddKernelNode(&kn, bodyg, nullptr, 0, &kp));
  cudaGraphExec_t ex;
  CK(cudaGraphInstantiate(&ex, graph, 0));
  for (int r = 0; r < runs; ++r) {
    Ctl c0 = {0u, 7u + (unsigned)r};
    CK(cudaMemcpyAsync(ctl, &c0, sizeof c0, cudaMemcpyHostToDevice, s));
    CK(cudaGraphLaunch(ex, s));
    Ctl c1;
    CK(cudaMemcpyAsync(&c1, ctl, sizeof c1, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    std::printf("run %d: iter %u (expect %u)\n", r, c1.iter, c0.max_iters);
    if (c1.iter != c0.max_iters) return 2;
  }
  std::printf("ok\n");
  return 0;
}
