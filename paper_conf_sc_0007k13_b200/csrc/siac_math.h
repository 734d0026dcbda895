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

}  // namespace siac
