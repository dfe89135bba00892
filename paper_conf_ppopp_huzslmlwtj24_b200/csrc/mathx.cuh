// fp64 tanh for the embedding nets' activations, written for the DFMA pipe.
//   tanh(x) = sign(x) t / (t + 2),  t = expm1(2|x|)
//   expm1(y) = 2^n (1 + p(f)) - 1,  y = n ln2 + f, |f| <= ln2/2, p = expm1 Taylor polynomial to f^12
//   (truncation < 5e-16 relative), so the small-|x| branch (n = 0) keeps full relative accuracy; the
//   quotient is the correctly rounded reciprocal refined by one residual step.  2|x| is clamped at 40
//   (1 - tanh(20) < 2^-56, so the result rounds to sign(x)).  About 30 fp64 instructions against ~130 issued for the libdevice tanh.
#pragma once

namespace fekf {

// Coefficients live in the constant bank so every DFMA takes them as a c[][] operand (64-bit literals
// would cost two uniform moves per use).
static __constant__ double c_tanh_k[16] = {
    2.08767569878680989792e-09, 2.50521083854417187751e-08, 2.75573192239858906526e-07,
    2.75573192239858906526e-06, 2.48015873015873015873e-05, 1.98412698412698412698e-04,
    1.38888888888888888889e-03, 8.33333333333333333333e-03, 4.16666666666666666667e-02,
    1.66666666666666666667e-01, 0.5,                        1.4426950408889634,
    6.93147180369123816490e-01, 1.90821492927058770002e-10, 6755399441055744.0, 0.0};

__device__ __forceinline__ double tanh_fp64(double x) {
  // branch-free (so a thread's independent tanh chains interleave): 2|x| is clamped at 40, where
  // t / (t + 2) rounds to 1; NaN passes through the select
  const double y0 = 2.0 * fabs(x);
  const double y = y0 > 40.0 ? 40.0 : y0;
  const double magic = c_tanh_k[14];                   // 1.5 * 2^52: round-to-nearest in the low word
  const double kd = fma(y, c_tanh_k[11], magic);
  const int n = __double2loint(kd);
  const double nd = kd - magic;
  double f = fma(-nd, c_tanh_k[12], y);                // ln2 hi
  f = fma(-nd, c_tanh_k[13], f);                       // ln2 lo
  double p = c_tanh_k[0];                              // 1/12! ... 1/2!
#pragma unroll
  for (int k = 1; k <= 10; ++k) p = fma(p, f, c_tanh_k[k]);
  p = fma(p * f, f, f);                                // expm1(f)
  const double scale = __hiloint2double((n + 1023) << 20, 0);
  const double t = fma(scale, p, scale - 1.0);         // expm1(y)
  const double den = t + 2.0;
  const double r = __drcp_rn(den);
  double q = t * r;
  q = fma(fma(-q, den, t), r, q);
  return copysign(q, x);
}

}  // namespace fekf
