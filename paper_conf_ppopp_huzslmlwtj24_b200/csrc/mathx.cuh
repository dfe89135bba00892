// fp64 tanh for the embedding and fitting nets' activations, written for the DFMA pipe.
//   tanh(x) = sign(x) t / (t + 2),  t = expm1(2|x|)
//   expm1(y) = 2^n T_j (1 + p(r)) - 1,  y = (64 n + j) ln2/64 + r,  |r| <= ln2/128,
//   T_j = 2^(j/64) as a hi + lo pair (table; lo of j = 0 is 2^-1000 instead of 0, so 2^n is applied to both
//   by an exponent add), p = expm1 Taylor polynomial to r^6 (truncation < 2e-20),
//   t = fma(S_hi, p, S_hi - 1) + S_lo (1 + p): no cancellation error for small y (S_hi - 1 is exact and
//   the table's rounding is carried by S_lo).  The quotient: one Newton step from rcp.approx, then one
//   residual correction of q.  2|x| is clamped at 40 (1 - tanh(20) < 2^-56).  Max relative error about
//   2 ulp (emulated against 50-digit decimal arithmetic: 4.7e-16); 20 fp64-pipe instructions: |x| and the
//   clamp on the integer side, the factor 2 of 2|x| folded into the constants (the previous single-interval
//   degree-12 version cost 36 DFMA lane-op equivalents in tools/fp64_mix.cu).
#pragma once

namespace fekf {

__device__ __align__(16) static const double2 g_exp2_tab[64] = {
    {1.0, 9.332636185032189e-302},
    {1.0108892860517005, -1.5234778603368577e-17},
    {1.0218971486541166, 5.109225028973444e-17},
    {1.0330248790212284, 7.600838874027088e-18},
    {1.0442737824274138, 8.551889705537965e-17},
    {1.0556451783605572, 1.759325738772092e-18},
    {1.0671404006768237, -7.899853966841582e-17},
    {1.0787607977571199, -6.656660436056593e-17},
    {1.0905077326652577, -3.046782079812471e-17},
    {1.102382583307841, 5.2660368715706944e-17},
    {1.1143867425958924, 1.0410278456845571e-16},
    {1.1265216186082418, 5.165856758795457e-17},
    {1.1387886347566916, 8.912812676025408e-17},
    {1.1511892299529827, 3.250710218863827e-17},
    {1.1637248587775775, 3.8292048369240935e-17},
    {1.1763969916502812, 5.554203254218079e-17},
    {1.189207115002721, 3.982015231465646e-17},
    {1.202156731452703, 6.644981499252301e-17},
    {1.215247359980469, -7.712630692681488e-17},
    {1.22848053610687, -1.89878163130253e-17},
    {1.241857812073484, 4.658027591836937e-17},
    {1.255380757024691, -6.7113898212968784e-18},
    {1.2690509571917332, 2.667932131342186e-18},
    {1.2828700160787783, 1.713594918243561e-17},
    {1.2968395546510096, 2.5382502794888315e-17},
    {1.3109612115247644, -7.181536135519454e-17},
    {1.3252366431597413, -2.8587312100388614e-17},
    {1.339667524053303, 8.927282594831732e-17},
    {1.3542555469368927, 7.70094837980299e-17},
    {1.3690024229745905, 9.593797919118849e-17},
    {1.383909881963832, -6.770511658794786e-17},
    {1.3989796725383112, -9.614213209051323e-17},
    {1.4142135623730951, -9.667293313452913e-17},
    {1.42961333839197, -1.2031642489053655e-17},
    {1.4451808069770467, -3.0237581349939873e-17},
    {1.460917794180647, -5.600377186075216e-17},
    {1.4768261459394993, -3.483994556892796e-17},
    {1.4929077282912648, 1.4192920154284036e-17},
    {1.5091644275934228, -1.016455327754295e-16},
    {1.5255981507445384, -1.1024941712342561e-16},
    {1.5422108254079407, 7.949834809697621e-17},
    {1.559004400237837, 3.7812070533575275e-17},
    {1.5759808451078865, -1.0136916471278304e-17},
    {1.593142151342267, -1.0094406542311964e-16},
    {1.6104903319492543, 2.4707192569797888e-17},
    {1.6280274218573478, -6.712955084707084e-17},
    {1.645755478153965, -1.0125679913674773e-16},
    {1.6636765803267364, 5.8909926967131e-17},
    {1.681792830507429, 8.199010020581497e-17},
    {1.7001063537185235, -8.0237193703977e-18},
    {1.718619298122478, -1.851380418263111e-17},
    {1.7373338352737062, 3.164389299292957e-17},
    {1.7562521603732995, 2.960140695448873e-17},
    {1.7753764925265212, 6.429731796556572e-17},
    {1.7947090750031072, 1.8227458427912087e-17},
    {1.8142521755003989, -9.969531538920349e-17},
    {1.8340080864093424, 3.283107224245627e-17},
    {1.8539791250833855, 9.761887490727594e-17},
    {1.8741676341103, -6.122763413004143e-17},
    {1.8945759815869656, 3.4034035352165297e-17},
    {1.9152065613971474, -1.0619946056195963e-16},
    {1.9360617934922943, 1.0332385960676326e-16},
    {1.9571441241754002, 8.960767791036668e-17},
    {1.978456026387951, 4.0388753109278167e-17}
};

__device__ __forceinline__ double tanh_fp64(double x) {
  // a = |x| clamped at 20 on the integer side (2|x| = 40: 1 - tanh(20) < 2^-56; NaN stays NaN)
  const int xh = __double2hiint(x) & 0x7fffffff;
  const double a = xh >= 0x40340000 && xh < 0x7ff00000 ? 20.0 : __hiloint2double(xh, __double2loint(x));
  const double magic = 6755399441055744.0;             // 1.5 * 2^52: round-to-nearest in the low word
  const double kd = fma(a, 184.6649652337873, magic);  // 2|x| * 64 / ln2
  const int k = __double2loint(kd);
  const double nd = kd - magic;
  double r = fma(-nd, 0.0054152123630046844, a);   // ln2/128, high part (24 bits: exact product)
  r = fma(-nd, -1.4880111718420063e-11, r);          // ln2/128, low part: r = (2|x| - k ln2/64) / 2
  // expm1(2r) = 2r + (2r)^2 (1/2 + 2r/6 + (2r)^2/24 + (2r)^3/120 + (2r)^4/720), coefficients pre-scaled by 2^k
  double q = fma(r, 16.0 / 720.0, 8.0 / 120.0);
  q = fma(q, r, 4.0 / 24.0);
  q = fma(q, r, 2.0 / 6.0);
  q = fma(q, r, 0.5);
  const double p = fma(4.0 * r, r * q, 2.0 * r);       // expm1(2r)
  const double2 T = __ldg(&g_exp2_tab[k & 63]);
  const int e = (k >> 6) << 20;                        // 2^n into the exponent fields (T.y is never 0)
  const double sh = __hiloint2double(__double2hiint(T.x) + e, __double2loint(T.x));
  const double sl = __hiloint2double(__double2hiint(T.y) + e, __double2loint(T.y));
  double t = fma(sh, p, sh - 1.0);
  t = fma(sl, 1.0 + p, t);                             // expm1(2|x|)
  const double den = t + 2.0;
  double rc;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(rc) : "d"(den));
  rc = fma(rc, fma(-den, rc, 1.0), rc);                // one Newton step
  double qq = t * rc;
  qq = fma(fma(-qq, den, t), rc, qq);                  // residual correction
  return copysign(qq, x);
}

// the nets' activation in their own precision (real.cuh): fp64 above, fp32 the CUDA math library's tanhf
// (max 2 ulp)
__device__ __forceinline__ double tanh_r(double x) { return tanh_fp64(x); }
__device__ __forceinline__ float tanh_r(float x) { return tanhf(x); }

}  // namespace fekf
