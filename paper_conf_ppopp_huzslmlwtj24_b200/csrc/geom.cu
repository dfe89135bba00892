// (a1) neighbour list and (a2) smooth environment matrix — P:L83 (§2.1 item 1).
#include <math_constants.h>

#include "model.cuh"

namespace fekf {

constexpr int NL_CAP = 1024;     // candidates kept per atom before sorting
constexpr int NL_THREADS = 128;
constexpr int SHIFT_BASE = 15, SHIFT_OFF = 7;

__device__ __forceinline__ bool key_less(int ta, double ra, int ja, int sa, int tb, double rb, int jb, int sb) {
  if (ta != tb) return ta < tb;
  if (ra != rb) return ra < rb;
  if (ja != jb) return ja < jb;
  return sa < sb;
}

// cross(u, v) . w  and |cross(u, v)| — plain fp64
__device__ double face_spacing(const double* a, const double* b, const double* c, double vol) {
  // spacing of the lattice planes spanned by (b, c): V / |b x c|
  const double x = b[1] * c[2] - b[2] * c[1], y = b[2] * c[0] - b[0] * c[2], z = b[0] * c[1] - b[1] * c[0];
  return vol / sqrt(x * x + y * y + z * z);
}

// One CTA per (image, atom).  Every candidate (j, n) is tested with separately rounded fp64
// operations (no FMA contraction), kept candidates are ranked by the total order
// (type_j, r^2, j, shift_id) and scattered into their type section; extra neighbours are counted.
__global__ void __launch_bounds__(NL_THREADS)
nlist_kernel(const double* __restrict__ coord, const double* __restrict__ box, const int* __restrict__ types,
             int Na, int ntypes, const int* __restrict__ sel_d, const int* __restrict__ sec_d, int Nm,
             double rcut, double rc2, int* __restrict__ nl_j, int* __restrict__ nl_s, int* __restrict__ overflow,
             int* __restrict__ err_flag) {
  __shared__ double c_r2[NL_CAP];
  __shared__ int c_j[NL_CAP], c_s[NL_CAP], c_t[NL_CAP], c_rank[NL_CAP];
  __shared__ int s_cnt, s_over, s_tcnt[FEKF_MAX_TYPES], s_m[3];
  __shared__ double s_box[9];
  const int b = blockIdx.x / Na, i = blockIdx.x % Na;
  const int tid = threadIdx.x;
  if (tid < 9) s_box[tid] = box[(size_t)b * 9 + tid];
  if (tid == 0) { s_cnt = 0; s_over = 0; }
  if (tid < FEKF_MAX_TYPES) s_tcnt[tid] = 0;
  __syncthreads();
  if (tid == 0) {
    const double* A = s_box;
    const double* B = s_box + 3;
    const double* C = s_box + 6;
    const double cx = B[1] * C[2] - B[2] * C[1], cy = B[2] * C[0] - B[0] * C[2], cz = B[0] * C[1] - B[1] * C[0];
    const double vol = fabs(A[0] * cx + A[1] * cy + A[2] * cz);
    s_m[0] = (int)ceil(rcut / face_spacing(A, B, C, vol));
    s_m[1] = (int)ceil(rcut / face_spacing(B, C, A, vol));
    s_m[2] = (int)ceil(rcut / face_spacing(C, A, B, vol));
  }
  __syncthreads();
  const int ma = s_m[0], mb = s_m[1], mc = s_m[2];
  if (ma > SHIFT_OFF || mb > SHIFT_OFF || mc > SHIFT_OFF) {
    // periodic images beyond the shift-id encoding (|n| <= 7; r_c more than 7 face spacings): the list is
    // left empty and the fault flag raised (metrics[7] bit 2) instead of mis-decoded shifts
    if (tid == 0) atomicOr(err_flag, 2);
    int* oj = nl_j + ((size_t)b * Na + i) * Nm;
    int* os = nl_s + ((size_t)b * Na + i) * Nm;
    for (int p = tid; p < Nm; p += NL_THREADS) { oj[p] = -1; os[p] = -1; }
    return;
  }
  const int na_ = 2 * ma + 1, nb_ = 2 * mb + 1, nc_ = 2 * mc + 1;
  const long long nshift = (long long)na_ * nb_ * nc_;
  const double* xi = coord + ((size_t)b * Na + i) * 3;
  const double xi0 = xi[0], xi1 = xi[1], xi2 = xi[2];
  // shifts outer (uniform over the CTA: no per-candidate integer division), atoms j strided over threads
  for (long long sidx = 0; sidx < nshift; ++sidx) {
    const int ic = (int)(sidx % nc_) - mc;
    const int ib = (int)((sidx / nc_) % nb_) - mb;
    const int ia = (int)(sidx / ((long long)nc_ * nb_)) - ma;
    const double fa = (double)ia, fb = (double)ib, fc = (double)ic;
    double S[3];
#pragma unroll
    for (int ax = 0; ax < 3; ++ax)
      S[ax] = __dadd_rn(__dadd_rn(__dmul_rn(fa, s_box[ax]), __dmul_rn(fb, s_box[3 + ax])), __dmul_rn(fc, s_box[6 + ax]));
    const int sid = ((ia + SHIFT_OFF) * SHIFT_BASE + (ib + SHIFT_OFF)) * SHIFT_BASE + (ic + SHIFT_OFF);
    const bool self_shift = ia == 0 && ib == 0 && ic == 0;
    for (int j = tid; j < Na; j += NL_THREADS) {
      if (j == i && self_shift) continue;
      const double* xj = coord + ((size_t)b * Na + j) * 3;
      const double dx = __dadd_rn(__dsub_rn(xj[0], xi0), S[0]);
      const double dy = __dadd_rn(__dsub_rn(xj[1], xi1), S[1]);
      const double dz = __dadd_rn(__dsub_rn(xj[2], xi2), S[2]);
      const double r2 = __dadd_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)), __dmul_rn(dz, dz));
      if (r2 < rc2) {
        const int pos = atomicAdd(&s_cnt, 1);
        if (pos < NL_CAP) {
          c_r2[pos] = r2;
          c_j[pos] = j;
          c_s[pos] = sid;
          c_t[pos] = types[j];
        }
      }
    }
  }
  __syncthreads();
  int cnt = s_cnt;
  if (cnt > NL_CAP) {
    if (tid == 0) atomicOr(err_flag, 1);
    cnt = NL_CAP;
  }
  for (int e = tid; e < cnt; e += NL_THREADS) {
    int rk = 0;
    const int te = c_t[e], je = c_j[e], se = c_s[e];
    const double re = c_r2[e];
    for (int f = 0; f < cnt; ++f) rk += key_less(c_t[f], c_r2[f], c_j[f], c_s[f], te, re, je, se) ? 1 : 0;
    c_rank[e] = rk;
    atomicAdd(&s_tcnt[te], 1);
  }
  __syncthreads();
  int* oj = nl_j + ((size_t)b * Na + i) * Nm;
  int* os = nl_s + ((size_t)b * Na + i) * Nm;
  for (int e = tid; e < cnt; e += NL_THREADS) {
    const int t = c_t[e];
    int start = 0;
    for (int u = 0; u < t; ++u) start += s_tcnt[u];
    const int pos = c_rank[e] - start;
    if (pos < sel_d[t]) {
      oj[sec_d[t] + pos] = c_j[e];
      os[sec_d[t] + pos] = c_s[e];
    } else {
      atomicAdd(&s_over, 1);
    }
  }
  for (int t = 0; t < ntypes; ++t)
    for (int p = s_tcnt[t] + tid; p < sel_d[t]; p += NL_THREADS) {
      oj[sec_d[t] + p] = -1;
      os[sec_d[t] + p] = -1;
    }
  __syncthreads();
  if (tid == 0 && s_over > 0) atomicAdd(&overflow[b], s_over);
}

// R~ row s(r)(1, d/r), J = dR~/dd (4x3) and d for every slot; zeros for padding.
// s(r) = sw(u)/r, u = (r - r_cs)/(r_c - r_cs), sw = 1 (r < r_cs), u^3(-6u^2+15u-10)+1 (reading Z8).
// switch_kind 1: sw = 0.5 cos(pi u) + 0.5.  stats [2][ntypes][4] (avg | std, reading Z11): valid rows of
// a centre atom of type t become (row - avg[t]) / std[t], J rows / std[t].
__global__ void envmat_kernel(const double* __restrict__ coord, const double* __restrict__ box,
                              const int* __restrict__ nl_j, const int* __restrict__ nl_s, int Na, int Nm,
                              long long nslots, double rcut, double rcs, int switch_kind,
                              const int* __restrict__ types, const double* __restrict__ stats, int ntypes,
                              double* __restrict__ em, double* __restrict__ jac, double* __restrict__ rij) {
  const long long idx = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= nslots) return;
  const int j = nl_j[idx];
  double* o_em = em + idx * 4;
  double* o_j = jac + idx * 12;
  double* o_d = rij + idx * 3;
  if (j < 0) {
#pragma unroll
    for (int k = 0; k < 4; ++k) o_em[k] = 0.0;
#pragma unroll
    for (int k = 0; k < 12; ++k) o_j[k] = 0.0;
#pragma unroll
    for (int k = 0; k < 3; ++k) o_d[k] = 0.0;
    return;
  }
  const long long bi = idx / Nm;
  const int b = (int)(bi / Na);
  const int sid = nl_s[idx];
  const int ic = sid % SHIFT_BASE - SHIFT_OFF;
  const int ib = (sid / SHIFT_BASE) % SHIFT_BASE - SHIFT_OFF;
  const int ia = sid / (SHIFT_BASE * SHIFT_BASE) - SHIFT_OFF;
  const double* bx = box + (size_t)b * 9;
  const double* xi = coord + bi * 3;
  const double* xj = coord + ((size_t)b * Na + j) * 3;
  double d[3];
#pragma unroll
  for (int ax = 0; ax < 3; ++ax) {
    const double S = __dadd_rn(__dadd_rn(__dmul_rn((double)ia, bx[ax]), __dmul_rn((double)ib, bx[3 + ax])),
                               __dmul_rn((double)ic, bx[6 + ax]));
    d[ax] = __dadd_rn(__dsub_rn(xj[ax], xi[ax]), S);
  }
  const double r2 = __dadd_rn(__dadd_rn(__dmul_rn(d[0], d[0]), __dmul_rn(d[1], d[1])), __dmul_rn(d[2], d[2]));
  const double r = sqrt(r2);
  double sw, dsw;
  if (r < rcs) {
    sw = 1.0;
    dsw = 0.0;
  } else if (r < rcut) {
    const double h = rcut - rcs;
    const double u = (r - rcs) / h;
    if (switch_kind == 1) {
      double sp, cp;
      sincospi(u, &sp, &cp);
      sw = 0.5 * cp + 0.5;
      dsw = -0.5 * CUDART_PI * sp / h;
    } else {
      sw = u * u * u * (-6.0 * u * u + 15.0 * u - 10.0) + 1.0;
      dsw = (-30.0 * u * u * u * u + 60.0 * u * u * u - 30.0 * u * u) / h;
    }
  } else {
    sw = 0.0;
    dsw = 0.0;
  }
  const double s = sw / r;
  const double ds = dsw / r - sw / r2;   // d s / d r
  const double ir = 1.0 / r;
  const double e[3] = {d[0] * ir, d[1] * ir, d[2] * ir};
  const double* avg = stats + types[bi % Na] * 4;
  const double* sd = stats + (ntypes + types[bi % Na]) * 4;
  o_em[0] = (s - avg[0]) / sd[0];
  o_em[1] = (s * d[0] / r - avg[1]) / sd[1];
  o_em[2] = (s * d[1] / r - avg[2]) / sd[2];
  o_em[3] = (s * d[2] / r - avg[3]) / sd[3];
#pragma unroll
  for (int be = 0; be < 3; ++be) o_j[be] = ds * e[be] / sd[0];
#pragma unroll
  for (int a = 0; a < 3; ++a)
#pragma unroll
    for (int be = 0; be < 3; ++be)
      o_j[3 * (a + 1) + be] = (ds * e[be] * e[a] + s * ((a == be ? ir : 0.0) - e[a] * e[be] * ir)) / sd[a + 1];
#pragma unroll
  for (int k = 0; k < 3; ++k) o_d[k] = d[k];
}

fekf_status launch_nlist(Ctx& c, const double* coord, const double* box, int nb, int* nl_j, int* nl_s,
                         int* overflow, cudaStream_t s) {
  FEKF_CHECK_CUDA(cudaMemsetAsync(overflow, 0, sizeof(int) * nb, s));
  const double rc2 = c.m.rcut * c.m.rcut;
  nlist_kernel<<<nb * c.Na, NL_THREADS, 0, s>>>(coord, box, c.types_d.as<int>(), c.Na, c.m.ntypes, c.sel_d.as<int>(),
                                                c.sec_d.as<int>(), c.Nm, c.m.rcut, rc2, nl_j, nl_s, overflow,
                                                c.err_d.as<int>());
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

fekf_status launch_envmat(Ctx& c, const double* coord, const double* box, const int* nl_j, const int* nl_s, int nb,
                          double* em, double* jac, double* rij, cudaStream_t s) {
  const long long n = (long long)nb * c.Na * c.Nm;
  envmat_kernel<<<cdiv(n, 128), 128, 0, s>>>(coord, box, nl_j, nl_s, c.Na, c.Nm, n, c.m.rcut, c.m.rcut_smth,
                                              c.m.switch_kind, c.types_d.as<int>(), c.env_stats.as<double>(), c.nt,
                                              em, jac, rij);
  FEKF_LAUNCH_CHECK();
  count_launch();
  return FEKF_OK;
}

}  // namespace fekf
