// siac_math.h -- host-side exact constants (implemented in siac_math.cpp, compiled by g++).
#pragma once

#include <utility>
#include <vector>

namespace siac {

// K on kernel cell i (i = 0..3k) as sum_m T[i*(k+1)+m] tau^m, tau = t - (t_i + 1/2),
// t_i = -(3k+1)/2 + i; optionally also the 2k+1 kernel coefficients c_gamma.
std::vector<double> kernel_cell_table(int k, std::vector<double> *coeffs_out = nullptr);

// Row-major nb x nb: row i = orthonormal Dubiner mode i in centred monomials, device Horner order.
std::vector<double> dubiner_to_centred(int k, std::vector<std::pair<int, int>> *order_out = nullptr);

// One-sided kernels: B-spline pieces ((k+1) x (k+1), piece-major) and the inverse of the
// symmetric kernel's moment matrix ((2k+1)^2, row g = coefficient index); c(lambda) =
// ainv . ((-lambda)^m)_m (siac_math.cpp).
void onesided_tables(int k, std::vector<double> &pieces, std::vector<double> &ainv);

// Same layout for SIAC_BASIS_MONOMIAL_REF: row i = r^a s^b (i by n = a + b, then b) in the
// centred monomials (r = (rho + 1)/3, s = (sigma + 1)/3), exact rationals rounded once.
std::vector<double> monomial_to_centred(int k);

}  // namespace siac
