// svd.cpp -- host FP64 one-sided (Hestenes) Jacobi SVD for the rank-r
// variant (R7).  Rows of W (N x K) are rotated pairwise until
// mutually orthogonal: W' = Q^T W with Q orthogonal, then W = Q W' and
//   sigma_i = ||w'_i||,  v_i = w'_i / sigma_i,  u_i = Q[:, i].
// Pairs are visited in round-robin tournament order so every round's N/2
// rotations touch disjoint rows and run on worker threads.
// (The oracle uses a different algorithm -- Jacobi eigen-decomposition of the
// Gram matrix -- and shares no code with this file.)
#include <algorithm>
#include <cmath>
#include <thread>
#include <vector>

#include "svd.h"

namespace pcnn {

static void rotate_pair(std::vector<double> &W, std::vector<double> &Q, int n, int k,
                        int p, int q, double tol, int *rotated) {
  double *wp = &W[(size_t)p * k], *wq = &W[(size_t)q * k];
  double a = 0, b = 0, c = 0;
  for (int i = 0; i < k; ++i) {
    a += wp[i] * wp[i];
    b += wq[i] * wq[i];
    c += wp[i] * wq[i];
  }
  if (std::fabs(c) <= tol * std::sqrt(a * b) || c == 0.0) return;
  *rotated = 1;
  const double zeta = (b - a) / (2.0 * c);
  const double t = (zeta >= 0 ? 1.0 : -1.0) / (std::fabs(zeta) + std::sqrt(1.0 + zeta * zeta));
  const double cs = 1.0 / std::sqrt(1.0 + t * t), sn = cs * t;
  for (int i = 0; i < k; ++i) {
    const double x = wp[i], y = wq[i];
    wp[i] = cs * x - sn * y;
    wq[i] = sn * x + cs * y;
  }
  // Q <- Q J (columns p, q), Q is n x n row-major
  for (int r = 0; r < n; ++r) {
    const double x = Q[(size_t)r * n + p], y = Q[(size_t)r * n + q];
    Q[(size_t)r * n + p] = cs * x - sn * y;
    Q[(size_t)r * n + q] = sn * x + cs * y;
  }
}

Svd svd_rows(const std::vector<double> &Win, int n, int k) {
  std::vector<double> W = Win;
  std::vector<double> Q((size_t)n * n, 0.0);
  for (int i = 0; i < n; ++i) Q[(size_t)i * n + i] = 1.0;
  const int m = n + (n & 1);                 // tournament size (even)
  std::vector<int> ring(m);
  for (int i = 0; i < m; ++i) ring[i] = i;
  const int nthreads = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
  const double tol = 1e-15;
  for (int sweep = 0; sweep < 60; ++sweep) {
    int any = 0;
    for (int round = 0; round < m - 1; ++round) {
      std::vector<std::pair<int, int>> pairs;
      for (int i = 0; i < m / 2; ++i) {
        int p = ring[i], q = ring[m - 1 - i];
        if (p >= n || q >= n) continue;
        if (p > q) std::swap(p, q);
        pairs.emplace_back(p, q);
      }
      std::vector<int> rot(nthreads, 0);
      // Q updates touch columns p,q of every row: disjoint pairs -> disjoint columns.
      auto work = [&](int tix) {
        for (size_t i = tix; i < pairs.size(); i += nthreads)
          rotate_pair(W, Q, n, k, pairs[i].first, pairs[i].second, tol, &rot[tix]);
      };
      if ((long long)pairs.size() * k < 20000 || nthreads == 1) {
        work(0);
        for (int t = 1; t < nthreads; ++t) work(t);
      } else {
        std::vector<std::thread> th;
        for (int t = 0; t < nthreads; ++t) th.emplace_back(work, t);
        for (auto &x : th) x.join();
      }
      for (int v : rot) any |= v;
      // rotate the ring (keep ring[0] fixed)
      const int last = ring[m - 1];
      for (int i = m - 1; i > 1; --i) ring[i] = ring[i - 1];
      ring[1] = last;
    }
    if (!any) break;
  }
  Svd s;
  s.n = n;
  s.k = k;
  std::vector<double> nrm(n);
  for (int i = 0; i < n; ++i) {
    double a = 0;
    for (int j = 0; j < k; ++j) a += W[(size_t)i * k + j] * W[(size_t)i * k + j];
    nrm[i] = std::sqrt(a);
  }
  std::vector<int> order(n);
  for (int i = 0; i < n; ++i) order[i] = i;
  std::stable_sort(order.begin(), order.end(), [&](int x, int y) { return nrm[x] > nrm[y]; });
  s.sigma.resize(n);
  s.U.assign((size_t)n * n, 0.0);
  s.Vt.assign((size_t)n * k, 0.0);
  for (int i = 0; i < n; ++i) {
    const int o = order[i];
    s.sigma[i] = nrm[o];
    for (int r = 0; r < n; ++r) s.U[(size_t)r * n + i] = Q[(size_t)r * n + o];
    const double inv = nrm[o] > 0 ? 1.0 / nrm[o] : 0.0;
    for (int j = 0; j < k; ++j) s.Vt[(size_t)i * k + j] = W[(size_t)o * k + j] * inv;
  }
  return s;
}

}  // namespace pcnn
