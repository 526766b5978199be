// svd.h -- host FP64 one-sided Jacobi SVD used by the rank-r variant (R7).
#pragma once
#include <vector>

namespace pcnn {

struct Svd {
  int n = 0, k = 0;
  std::vector<double> sigma;   // n, descending
  std::vector<double> U;       // n x n row-major; column i = u_i
  std::vector<double> Vt;      // n x k; row i = v_i^T
};

// SVD of the row-major n x k matrix W.
Svd svd_rows(const std::vector<double> &W, int n, int k);

}  // namespace pcnn
