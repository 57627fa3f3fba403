// Probe: can a CUDA graph IF node whose body is stream-captured hold the
// local-restart redo (copy kernel, cuBLAS DGEMM, cuSOLVER dpotrf)?
// nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/cgp tools/cond_graph_probe.cu -lcublas -lcusolver
#include <cublas_v2.h>
#include <cuda_runtime.h>
#include <cusolverDn.h>
#include <chrono>
#include <cstdio>
#include <vector>

#define CK(x)                                                                     \
  do {                                                                            \
    auto e_ = (x);                                                                \
    if (e_ != 0) {                                                                \
      printf("FAIL %s:%d %s -> %d\n", __FILE__, __LINE__, #x, (int)e_);           \
      return 1;                                                                   \
    }                                                                             \
  } while (0)

__global__ void set_cond(cudaGraphConditionalHandle h, const int* flag) { cudaGraphSetConditional(h, *flag > 0); }
__global__ void add1(double* x, int n) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) x[i] += 1.0;
}

int main() {
  const int n = 512;
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cublasHandle_t hb;
  CK(cublasCreate(&hb));
  CK(cublasSetStream(hb, s));
  cusolverDnHandle_t hs;
  CK(cusolverDnCreate(&hs));
  CK(cusolverDnSetStream(hs, s));
  double *A, *B, *C, *S, *work;
  int *flag, *info;
  CK(cudaMalloc(&A, n * n * 8));
  CK(cudaMalloc(&B, n * n * 8));
  CK(cudaMalloc(&C, n * n * 8));
  CK(cudaMalloc(&S, n * n * 8));
  CK(cudaMalloc(&flag, 4));
  CK(cudaMalloc(&info, 4));
  int lw = 0;
  CK(cusolverDnDpotrf_bufferSize(hs, CUBLAS_FILL_MODE_LOWER, n, S, n, &lw));
  CK(cudaMalloc(&work, (size_t)lw * 8));
  std::vector<double> h(n * n);
  for (int i = 0; i < n * n; ++i) h[i] = (i % 7) * 0.25 - 0.5;
  CK(cudaMemcpy(A, h.data(), n * n * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(B, h.data(), n * n * 8, cudaMemcpyHostToDevice));
  for (int i = 0; i < n * n; ++i) h[i] = (i % (n + 1) == 0) ? n + 1.0 : 0.5;
  std::vector<double> spd = h;

  for (int trial = 0; trial < 2; ++trial) {
    CK(cudaMemcpy(S, spd.data(), n * n * 8, cudaMemcpyHostToDevice));
    CK(cudaMemset(C, 0, n * n * 8));
    int fv = trial;
    CK(cudaMemcpy(flag, &fv, 4, cudaMemcpyHostToDevice));
    auto t0 = std::chrono::steady_clock::now();
    cudaGraph_t g;
    CK(cudaGraphCreate(&g, 0));
    cudaGraphConditionalHandle ch;
    CK(cudaGraphConditionalHandleCreate(&ch, g, 0, 0));
    // node 1: the kernel that sets the condition (captured into g)
    CK(cudaStreamBeginCaptureToGraph(s, g, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
    set_cond<<<1, 1, 0, s>>>(ch, flag);
    cudaStreamCaptureStatus cst;
    const cudaGraphNode_t* deps;
    size_t ndep;
    CK(cudaStreamGetCaptureInfo(s, &cst, nullptr, nullptr, &deps, &ndep));
    cudaGraphNodeParams cp = {};
    cp.type = cudaGraphNodeTypeConditional;
    cp.conditional.handle = ch;
    cp.conditional.type = cudaGraphCondTypeIf;
    cp.conditional.size = 1;
    cudaGraphNode_t cnode;
    CK(cudaGraphAddNode(&cnode, g, deps, ndep, &cp));
    CK(cudaStreamUpdateCaptureDependencies(s, &cnode, 1, cudaStreamSetCaptureDependencies));
    CK(cudaStreamEndCapture(s, &g));
    cudaGraph_t body = cp.conditional.phGraph_out[0];
    CK(cudaStreamBeginCaptureToGraph(s, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
    add1<<<64, 256, 0, s>>>(A, n * n);
    const double one = 1.0, zero = 0.0;
    CK(cublasDgemm(hb, CUBLAS_OP_N, CUBLAS_OP_T, n, n, n, &one, A, n, B, n, &zero, C, n));
    CK(cusolverDnDpotrf(hs, CUBLAS_FILL_MODE_LOWER, n, S, n, work, lw, info));
    CK(cudaStreamEndCapture(s, &body));
    cudaGraphExec_t ge;
    CK(cudaGraphInstantiate(&ge, g, 0));
    auto t1 = std::chrono::steady_clock::now();
    CK(cudaGraphLaunch(ge, s));
    CK(cudaStreamSynchronize(s));
    double c0, s0, a0;
    CK(cudaMemcpy(&c0, C, 8, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&s0, S, 8, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&a0, A, 8, cudaMemcpyDeviceToHost));
    printf("trial flag=%d: A[0]=%g C[0]=%g S[0]=%g (chol would be %g) build+inst %.1f us\n", fv, a0, c0, s0,
           sqrt(n + 1.0), std::chrono::duration<double, std::micro>(t1 - t0).count());
    CK(cudaGraphExecDestroy(ge));
    CK(cudaGraphDestroy(g));
  }
  printf("PROBE OK\n");
  return 0;
}
