// cusparse_phases.cu — cuSPARSE's generic SpGEMM (cusparseSpGEMM_workEstimation / compute / copy)
// on device CSR inputs, with CUDA events between its phases and the device memory high-water mark,
// for the paper's Fig. 5/6 breakdown and Fig. 4 memory comparison (
// SURVEY.md §8(f2)).  A comparator, not part of the library: built by scripts/cusparse_phases.py.
//
//   int cusp_spgemm(int64 m, k, n, nnzA, nnzB, idx64, fp64,
//                   a_rpt, a_col, a_val, b_rpt, b_col, b_val   (device; rpt/col int32 or int64),
//                   double out[8])
//   out: [0] work-estimation ms (incl. buffer 1 allocation)  [1] compute ms (incl. buffer 2)
//        [2] cudaMalloc of C ms  [3] copy ms  [4] total ms  [5] nnz(C)  [6] peak bytes above entry
//        [7] status (0 ok, else cusparseStatus_t / -cudaError)
#include <cuda_runtime.h>
#include <cusparse.h>

#include <cstdint>

namespace {
size_t used_now() {
  size_t fr = 0, tot = 0;
  cudaMemGetInfo(&fr, &tot);
  return tot - fr;
}
}  // namespace

extern "C" int cusp_spgemm(int64_t m, int64_t k, int64_t n, int64_t nnza, int64_t nnzb, int idx64, int fp64,
                           void* a_rpt, void* a_col, void* a_val, void* b_rpt, void* b_col, void* b_val,
                           double* out) {
  for (int i = 0; i < 8; ++i) out[i] = 0;
  cusparseHandle_t h;
  if (cusparseCreate(&h) != CUSPARSE_STATUS_SUCCESS) return out[7] = 1, 1;
  const cusparseIndexType_t it = idx64 ? CUSPARSE_INDEX_64I : CUSPARSE_INDEX_32I;
  const cudaDataType vt = fp64 ? CUDA_R_64F : CUDA_R_32F;
  cusparseSpMatDescr_t A, B, C;
  cusparseCreateCsr(&A, m, k, nnza, a_rpt, a_col, a_val, it, it, CUSPARSE_INDEX_BASE_ZERO, vt);
  cusparseCreateCsr(&B, k, n, nnzb, b_rpt, b_col, b_val, it, it, CUSPARSE_INDEX_BASE_ZERO, vt);
  cusparseCreateCsr(&C, m, n, 0, nullptr, nullptr, nullptr, it, it, CUSPARSE_INDEX_BASE_ZERO, vt);
  cusparseSpGEMMDescr_t d;
  cusparseSpGEMM_createDescr(&d);
  double one = 1.0, zero = 0.0;
  float onef = 1.f, zerof = 0.f;
  const void* alpha = fp64 ? (const void*)&one : (const void*)&onef;
  const void* beta = fp64 ? (const void*)&zero : (const void*)&zerof;
  const auto op = CUSPARSE_OPERATION_NON_TRANSPOSE;
  const auto alg = CUSPARSE_SPGEMM_DEFAULT;
  cudaEvent_t ev[5];
  for (auto& e : ev) cudaEventCreate(&e);
  const size_t base = used_now();
  size_t peak = 0;
  auto track = [&]() {
    const size_t u = used_now();
    if (u > base && u - base > peak) peak = u - base;
  };
  size_t s1 = 0, s2 = 0;
  void *buf1 = nullptr, *buf2 = nullptr, *c_rpt = nullptr, *c_col = nullptr, *c_val = nullptr;
  int st = 0;
  const size_t ib = idx64 ? 8 : 4, vb = fp64 ? 8 : 4;
  cudaDeviceSynchronize();
  cudaEventRecord(ev[0]);
  // C's row offsets are part of the result (allocated before the count, as cuSPARSE requires)
  cudaMalloc(&c_rpt, (m + 1) * ib);
  st = cusparseSpGEMM_workEstimation(h, op, op, alpha, A, B, beta, C, vt, alg, d, &s1, nullptr);
  if (!st) { cudaMalloc(&buf1, s1 ? s1 : 1); track(); }
  if (!st) st = cusparseSpGEMM_workEstimation(h, op, op, alpha, A, B, beta, C, vt, alg, d, &s1, buf1);
  cudaEventRecord(ev[1]);
  if (!st) st = cusparseSpGEMM_compute(h, op, op, alpha, A, B, beta, C, vt, alg, d, &s2, nullptr);
  if (!st) { cudaMalloc(&buf2, s2 ? s2 : 1); track(); }
  if (!st) st = cusparseSpGEMM_compute(h, op, op, alpha, A, B, beta, C, vt, alg, d, &s2, buf2);
  cudaEventRecord(ev[2]);
  int64_t cm = 0, cn = 0, cnnz = 0;
  if (!st) st = cusparseSpMatGetSize(C, &cm, &cn, &cnnz);
  if (!st) {
    cudaError_t e1 = cudaMalloc(&c_col, (cnnz ? cnnz : 1) * ib);
    cudaError_t e2 = cudaMalloc(&c_val, (cnnz ? cnnz : 1) * vb);
    if (e1 != cudaSuccess || e2 != cudaSuccess) st = -(int)(e1 != cudaSuccess ? e1 : e2);
    track();
  }
  cudaEventRecord(ev[3]);
  if (!st) st = cusparseCsrSetPointers(C, c_rpt, c_col, c_val);
  if (!st) st = cusparseSpGEMM_copy(h, op, op, alpha, A, B, beta, C, vt, alg, d);
  cudaEventRecord(ev[4]);
  cudaError_t ce = cudaDeviceSynchronize();
  track();
  if (!st && ce != cudaSuccess) st = -(int)ce;
  float ms;
  for (int i = 0; i < 4; ++i) {
    cudaEventElapsedTime(&ms, ev[i], ev[i + 1]);
    out[i] = ms;
  }
  cudaEventElapsedTime(&ms, ev[0], ev[4]);
  out[4] = ms;
  out[5] = (double)cnnz;
  out[6] = (double)peak;
  out[7] = st;
  cudaFree(buf1); cudaFree(buf2); cudaFree(c_rpt); cudaFree(c_col); cudaFree(c_val);
  cusparseSpGEMM_destroyDescr(d);
  cusparseDestroySpMat(A); cusparseDestroySpMat(B); cusparseDestroySpMat(C);
  for (auto& e : ev) cudaEventDestroy(e);
  cusparseDestroy(h);
  return st;
}
