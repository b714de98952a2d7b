// Time of the dataflow POTRF (potrf_df) on one b x b SPD tile for a given
// grid (development tool, not the product).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Iinclude -Ipaper_conf_icpp_shenvms15_b200/csrc
//      -o tools/pp tools/potrf_probe.cu -lcuda
#include "../paper_conf_icpp_shenvms15_b200/csrc/kernels_chol.cu"
#include <cstdio>
#include <vector>

int main(int argc, char** argv) {
  const int grid = argc > 1 ? atoi(argv[1]) : 148;
  const int b = argc > 2 ? atoi(argv[2]) : 1024;
  std::vector<float> h((size_t)b * b);
  for (int i = 0; i < b; ++i)
    for (int j = 0; j < b; ++j) h[(size_t)i * b + j] = i == j ? (float)b : 0.5f * (float)((i * 7 + j * 13) % 17) / 17.f;
  for (int i = 0; i < b; ++i)
    for (int j = 0; j < i; ++j) h[(size_t)j * b + i] = h[(size_t)i * b + j];
  float* d;
  int* f;
  cudaMalloc(&d, h.size() * 4);
  cudaMalloc(&f, mm::chol_potrf_flag_bytes(b));
  for (int rep = 0; rep < 3; ++rep) {
    cudaMemcpy(d, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    cudaMemset(f, 0, mm::chol_potrf_flag_bytes(b));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    mm::potrf_df<<<grid, mm::kPfThreads>>>(d, b, f);
    cudaEventRecord(e1);
    cudaError_t e = cudaDeviceSynchronize();
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    printf("b=%d grid=%d rep %d: %s %.3f ms\n", b, grid, rep, cudaGetErrorString(e), ms);
  }
  return 0;
}
// stubs for the tensor-core entry points chol_batch references (unused here)
namespace mm {
size_t chol_tc_scratch(int64_t, int64_t) { return 0; }
cudaError_t chol_trsm_prepare(float*, int64_t, int64_t, int32_t, cudaStream_t, Scratch*, float**, float**, int32_t*) {
  return cudaErrorNotSupported;
}
void chol_mark_split(Scratch*, int64_t, int32_t, const int32_t*, int32_t) {}
cudaError_t chol_trsm_update_tc(float*, int64_t, int64_t, int32_t, const int32_t*, int32_t, int32_t, int32_t, int32_t,
                                cudaStream_t, Scratch*, bool) {
  return cudaErrorNotSupported;
}
}  // namespace mm
