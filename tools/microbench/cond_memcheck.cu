// Minimal repro for the open sanitizer item (DESIGN.md §8 "Sanitizers"):
// does compute-sanitizer memcheck fail a CUDA-graph conditional WHILE node
// whose body kernel sets the condition from device code, with none of the
// shard-pass code involved?
//   nvcc -gencode arch=compute_100a,code=sm_100a -o cond_memcheck cond_memcheck.cu -lcudadevrt -rdc=true
//   ./cond_memcheck [runs] [pad] [async] [iters]; compute-sanitizer --tool memcheck ./cond_memcheck [runs] [pad]
// `pad` = 1 passes a large by-value parameter struct (like the shard pass's KParams);
// `pad` = 2 runs the TMA/mbarrier/last-CTA body below.
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

// mode 2: like the shard pass — 200 KB dynamic shared memory, an mbarrier-completed
// cp.async.bulk of a global tile into it, and the LAST CTA to finish sets the condition.
struct Tma { Ctl* ctl; const float* src; float* dst; unsigned* done; cudaGraphConditionalHandle h; };
__global__ void body_tma(Tma p) {
  extern __shared__ __align__(128) unsigned char sm[];
  unsigned long long* bar = reinterpret_cast<unsigned long long*>(sm);
  float* tile = reinterpret_cast<float*>(sm + 128);
  const unsigned b = (unsigned)__cvta_generic_to_shared(bar), t = (unsigned)__cvta_generic_to_shared(tile);
  const unsigned bytes = 4096 * 4;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(t), "l"(p.src + (size_t)blockIdx.x * 4096), "r"(bytes), "r"(b) : "memory");
  }
  unsigned ok = 0;
  while (!ok)
    asm volatile("{\n .reg .pred q;\n mbarrier.try_wait.parity.shared::cta.b64 q, [%1], 0;\n selp.u32 %0, 1, 0, q;\n}\n"
                 : "=r"(ok) : "r"(b) : "memory");
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) p.dst[(size_t)blockIdx.x * 4096 + i] = tile[i] + 1.f;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(p.done, 1u) == gridDim.x - 1) {
      *p.done = 0;
      const unsigned n = ++p.ctl->iter;
      __threadfence();
      cudaGraphSetConditional(p.h, n < p.ctl->max_iters ? 1u : 0u);
    }
  }
}

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  std::printf("%s:%d %s -> %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); return 1; } } while (0)

int main(int argc, char** argv) {
  const int runs = argc > 1 ? std::atoi(argv[1]) : 5;
  const int big = argc > 2 ? std::atoi(argv[2]) : 0;
  // argv[3] = 1: a non-blocking stream and stream-ordered (cudaMallocAsync) buffers, as cusha_run uses
  const bool async = argc > 3 && std::atoi(argv[3]) == 1;
  cudaStream_t s;
  CK(async ? cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) : cudaStreamCreate(&s));
  Ctl* ctl;
  CK(async ? cudaMallocAsync(&ctl, sizeof(Ctl), s) : cudaMalloc(&ctl, sizeof(Ctl)));
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
  const int G = 148 * 1;
  const size_t smem = 200 * 1024;
  float *src, *dst;
  unsigned* done;
  if (async) {
    CK(cudaMallocAsync(&src, (size_t)G * 4096 * 4, s));
    CK(cudaMallocAsync(&dst, (size_t)G * 4096 * 4, s));
    CK(cudaMallocAsync(&done, 4, s));
  } else {
    CK(cudaMalloc(&src, (size_t)G * 4096 * 4));
    CK(cudaMalloc(&dst, (size_t)G * 4096 * 4));
    CK(cudaMalloc(&done, 4));
  }
  CK(cudaMemsetAsync(src, 0, (size_t)G * 4096 * 4, s));
  CK(cudaMemsetAsync(done, 0, 4, s));
  CK(cudaStreamSynchronize(s));
  CK(cudaFuncSetAttribute(body_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  Tma tp = {ctl, src, dst, done, h};
  void* args_tma[] = {&tp};
  Big bp = {};
  bp.ctl = ctl;
  bp.h = h;
  void* args_small[] = {&ctl, &h};
  void* args_big[] = {&bp};
  cudaKernelNodeParams kp = {};
  kp.func = big == 2 ? (void*)body_tma : big ? (void*)body_big : (void*)body_small;
  kp.gridDim = dim3(G);
  kp.blockDim = dim3(256);
  kp.sharedMemBytes = big == 2 ? (unsigned)smem : 0u;
  kp.kernelParams = big == 2 ? args_tma : big ? args_big : args_small;
  cudaGraphNode_t kn;
  CK(cudaGraphAddKernelNode(&kn, bodyg, nullptr, 0, &kp));
  cudaGraphExec_t ex;
  CK(cudaGraphInstantiate(&ex, graph, 0));
  for (int r = 0; r < runs; ++r) {
    // argv[4]: iterations per run (default 7), so a run can still be looping on the
    // device when the host issues its next API call
    const unsigned base = argc > 4 ? (unsigned)std::atoi(argv[4]) : 7u;
    Ctl c0 = {0u, base + (unsigned)r};
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
