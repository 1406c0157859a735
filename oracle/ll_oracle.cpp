// CPU ORACLE (C++17 + OpenMP) for the Linear Layouts conversion hot path —
// TEST INFRASTRUCTURE ONLY.
//
// Only tests/, __graft_entry__.smoke()/build() and bench.py's cpu_baseline /
// --impl reference legs may load this library (oracle/cpp.py).  It is built as its own
// shared object (oracle/libll_oracle.so), never linked into the product's libll.so, and
// shares no code, header, table or helper with the product.  It is the C++ twin of
// oracle/ll_oracle.py ("one plain C++17 file with OpenMP plus a Python
// mirror") and is cross-checked against it element by element (tests/test_oracle_cpp.py).
//
// Plain and slow on purpose: every layout evaluation is the XOR of the columns of the
// set bits, bit by bit (O2); no SIMD intrinsics, no blocking, no tables beyond the
// right inverse.  Citations P:L are lines of the paper's text.
//
// Conventions: a layout is given as its columns cols[k] = the logical
// flat index of input bit k (input dims in declaration order, first dim least
// significant; logical flat index row-major, last out dim fastest).
// A buffer packed in layout L holds at position h the logical element L(h).
#include <cstdint>
#include <cstring>
#include <vector>

#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

// O2 apply ("Bitwise XOR of these three coordinate pairs yields the
// register's absolute position"; w = Av over F2).
inline uint64_t apply(const uint64_t* cols, int d_in, uint64_t h) {
  uint64_t x = 0;
  for (int k = 0; k < d_in; ++k)
    if ((h >> k) & 1) x ^= cols[k];
  return x;
}

// O4 right inverse (Def 4.5): solve M X = I by Gaussian elimination, pivots
// over the columns of M in ascending order, free variables = 0 (the slack variables
// "set to zeros").  hcols[t] = hardware index X e_t for logical bit t.
bool right_inverse(const uint64_t* cols, int d_in, int d_out, uint64_t* hcols) {
  std::vector<uint64_t> pv(64, 0), pc(64, 0);
  std::vector<char> have(64, 0);
  for (int k = 0; k < d_in; ++k) {
    uint64_t v = cols[k], comb = uint64_t(1) << k;
    while (v) {
      const int lead = 63 - __builtin_clzll(v);
      if (!have[lead]) { have[lead] = 1; pv[lead] = v; pc[lead] = comb; break; }
      v ^= pv[lead];
      comb ^= pc[lead];
    }
  }
  for (int t = 0; t < d_out; ++t) if (!have[t]) return false;   // not surjective
  for (int t = 0; t < d_out; ++t) {
    uint64_t v = uint64_t(1) << t, comb = 0;
    while (v) {
      const int lead = 63 - __builtin_clzll(v);
      v ^= pv[lead];
      comb ^= pc[lead];
    }
    hcols[t] = comb;
  }
  return true;
}

void set_threads(int nthreads) {
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#else
  (void)nthreads;
#endif
}

}  // namespace

extern "C" {

int llo_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

// O2 over an array: xs[i] = L(hs[i]).
void llo_apply(const uint64_t* cols, int d_in, const uint64_t* hs, uint64_t* xs, int64_t n, int nthreads) {
  set_threads(nthreads);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) xs[i] = apply(cols, d_in, hs[i]);
}

// O4: the slack-zero right inverse's columns (returns 0, or -1 if L is not surjective).
int llo_right_inverse(const uint64_t* cols, int d_in, int d_out, uint64_t* hcols) {
  return right_inverse(cols, d_in, d_out, hcols) ? 0 : -1;
}

// O4 brute force: first[x] = min{h : L(h) = x}, scanning h ascending (small layouts).
int llo_preimage_min(const uint64_t* cols, int d_in, int d_out, int64_t* first) {
  const uint64_t nx = uint64_t(1) << d_out;
  for (uint64_t x = 0; x < nx; ++x) first[x] = -1;
  for (uint64_t h = 0; h < (uint64_t(1) << d_in); ++h) {
    const uint64_t x = apply(cols, d_in, h);
    if (first[x] < 0) first[x] = int64_t(h);
  }
  for (uint64_t x = 0; x < nx; ++x) if (first[x] < 0) return -1;
  return 0;
}

// O5 conversion, pull form of B^-1∘A:
//   dst[i] = src[A^+(B(h0 + i))]  for i in [0, n),
// B(h) evaluated bit by bit, A^+ applied linearly from its right-inverse columns.
// src is the whole buffer packed in A (2^dA elements of w bytes).
int llo_convert(const uint64_t* colsA, int dA, const uint64_t* colsB, int dB, int d_out, int w,
                const void* src, void* dst, uint64_t h0, int64_t n, int nthreads) {
  std::vector<uint64_t> inv(d_out);
  if (!right_inverse(colsA, dA, d_out, inv.data())) return -1;
  set_threads(nthreads);
  const uint8_t* s = static_cast<const uint8_t*>(src);
  uint8_t* d = static_cast<uint8_t*>(dst);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    const uint64_t x = apply(colsB, dB, h0 + uint64_t(i));
    const uint64_t hs = apply(inv.data(), d_out, x);
    std::memcpy(d + uint64_t(i) * w, s + hs * w, size_t(w));
  }
  return 0;
}

// O10 gather along an axis: src, idx and dst are packed in the same
// layout L.  For dst position h with logical x = L(h): the axis coordinate's
// low kbits bits (the in-tile part, K = 2^kbits) are replaced by idx[h] & (K-1)
// (out-of-range indices masked, G16), and dst[h] = src[L^+(x')].
int llo_gather(const uint64_t* cols, int d, int d_out, int axis_shift, int kbits, int w,
               const void* src, const int32_t* idx, void* dst, int nthreads) {
  std::vector<uint64_t> inv(d_out);
  if (!right_inverse(cols, d, d_out, inv.data())) return -1;
  set_threads(nthreads);
  const uint64_t kmask = ((uint64_t(1) << kbits) - 1) << axis_shift;
  const uint8_t* s = static_cast<const uint8_t*>(src);
  uint8_t* o = static_cast<uint8_t*>(dst);
  const int64_t n = int64_t(1) << d;
#pragma omp parallel for schedule(static)
  for (int64_t h = 0; h < n; ++h) {
    const uint64_t x = apply(cols, d, uint64_t(h));
    const uint64_t q = uint64_t(uint32_t(idx[h])) & ((uint64_t(1) << kbits) - 1);
    const uint64_t xs = (x & ~kmask) | (q << axis_shift);
    std::memcpy(o + uint64_t(h) * w, s + apply(inv.data(), d_out, xs) * w, size_t(w));
  }
  return 0;
}

// O11 reduce (sum) along an axis inside each tile (Table 4).
// The output is the logical tensor with the axis coordinate a replaced by a >> kbits,
// row-major: out[y], y = ((upper * (na >> kbits)) + (a >> kbits)) * 2^axis_shift + lower.
// fp64: plain sum.  fp32: the fixed order of reading R-reduce — for in-tile logical
// axis bit t = 0, 1, ... ascending, v <- v(t = 0) + v(t = 1) (round to nearest, no FMA;
// compiled without -ffast-math and with -ffp-contract=off).
static int reduce_common(const uint64_t* cols, int d, int d_out, int axis_shift, int axis_bits, int kbits,
                         const float* src, float* out32, double* out64, int nthreads) {
  std::vector<uint64_t> inv(d_out);
  if (!right_inverse(cols, d, d_out, inv.data())) return -1;
  set_threads(nthreads);
  const int64_t K = int64_t(1) << kbits;
  const int64_t n_out = int64_t(1) << (d_out - kbits);
  const uint64_t lower_mask = (uint64_t(1) << axis_shift) - 1;
  const int ob = axis_bits - kbits;   // output axis bits
#pragma omp parallel for schedule(static)
  for (int64_t y = 0; y < n_out; ++y) {
    const uint64_t lower = uint64_t(y) & lower_mask;
    const uint64_t a_hi = (uint64_t(y) >> axis_shift) & ((uint64_t(1) << ob) - 1);
    const uint64_t upper = uint64_t(y) >> (axis_shift + ob);
    std::vector<float> v32(K);
    double acc = 0.0;
    for (int64_t q = 0; q < K; ++q) {
      const uint64_t a = (a_hi << kbits) | uint64_t(q);
      const uint64_t x = (((upper << axis_bits) | a) << axis_shift) | lower;
      const float val = src[apply(inv.data(), d_out, x)];
      v32[q] = val;
      acc += double(val);
    }
    if (out64) out64[y] = acc;
    if (out32) {
      for (int t = 0; t < kbits; ++t) {
        const int64_t m = K >> (t + 1);
        for (int64_t q = 0; q < m; ++q) v32[q] = v32[2 * q] + v32[2 * q + 1];
      }
      out32[y] = v32[0];
    }
  }
  return 0;
}

int llo_reduce_fp32(const uint64_t* cols, int d, int d_out, int axis_shift, int axis_bits, int kbits,
                    const float* src, float* out, int nthreads) {
  return reduce_common(cols, d, d_out, axis_shift, axis_bits, kbits, src, out, nullptr, nthreads);
}

int llo_reduce_fp64(const uint64_t* cols, int d, int d_out, int axis_shift, int axis_bits, int kbits,
                    const float* src, double* out, int nthreads) {
  return reduce_common(cols, d, d_out, axis_shift, axis_bits, kbits, src, nullptr, out, nthreads);
}

}  // extern "C"
