/*
 * oracle/loops.c — CPU ORACLE for the loop nests on the CATT hot path.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code with paper_conf_icpp_kimhlsh19_b200/ (the CUDA path) and
 * includes none of its headers.
 *
 * What it computes: the plain textbook loop nests that CATT reschedules but
 * never changes (CATT "embeds a thread throttling code"; the
 * arithmetic of each loop is the original kernel's). Kernel bodies are the
 * PolyBench/GPU and Rodinia ones named in Table 2; ATAX kernel 1
 * is printed in Fig 1:   tmp[i] += A[i*NX + j] * B[j].
 *
 * Two modes, each a plain sequential loop per output (OpenMP only splits the
 * independent outputs; it never changes any output's order of operations):
 *   ORC_SEQ_FMAF (0): fp32, j (or i, k, f) ascending, acc = fmaf(a, b, acc)
 *       from the initial value. This is the literal loop as nvcc compiles it
 *       (a*b+c contracted to one fused multiply-add). Built with
 *       -ffp-contract=off so that only the explicit fmaf() calls fuse.
 *   ORC_SEQ_F64  (1): same order, double accumulation (inputs widened),
 *       rounded to fp32 once at the end; second-stage products use the
 *       unrounded double intermediate (the mathematically exact path).
 *
 * Also: the counter-based input generator, written independently of
 * seeded_inputs.py and of the CUDA generator (tests check all three agree).
 */
#include <float.h>
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { ORC_SEQ_FMAF = 0, ORC_SEQ_F64 = 1 };

/* ---------------------------------------------------------------- generator */
static uint32_t orc_fmix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85EBCA6Bu;
  h ^= h >> 13;
  h *= 0xC2B2AE35u;
  h ^= h >> 16;
  return h;
}

static uint32_t orc_hash(uint32_t seed, uint64_t idx) {
  uint32_t lo = (uint32_t)(idx & 0xFFFFFFFFu), hi = (uint32_t)(idx >> 32);
  uint32_t key = orc_fmix32(seed * 0x9E3779B9u + hi * 0x632BE5ABu + 0x7F4A7C15u);
  return orc_fmix32((lo * 0x85EBCA77u) ^ key);
}

static float orc_value(uint32_t seed, uint64_t idx, int mode) {
  uint32_t h = orc_hash(seed, idx);
  if (mode == 1) return (float)(h & 15u) * (1.0f / 16.0f);
  return (float)(h >> 8) * (1.0f / 16777216.0f);
}

/* out[k] = value(seed, offset + k) for k < n. */
void orc_fill(uint32_t seed, uint64_t offset, int64_t n, int mode, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t k = 0; k < n; ++k) out[k] = orc_value(seed, offset + (uint64_t)k, mode);
}

/* ---------------------------------------------------------------- ATAX
 * PolyBench/GPU atax (Table 2; Fig 1; Table 3):
 *   kernel 1 (row per thread, memory-divergent):  tmp[i] += A[i*n + j] * x[j]
 *   kernel 2 (column per thread, coalesced):      y[j]   += A[i*n + j] * tmp[i]
 * Outputs start at 0 (SURVEY 8(c) reading 13). A is m x n row-major. */
int orc_atax(int mode, const float* A, const float* x, float* tmp, float* y, int64_t m, int64_t n) {
  if (mode == ORC_SEQ_FMAF) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; ++i) {
      float acc = 0.0f;
      for (int64_t j = 0; j < n; ++j) acc = fmaf(A[i * n + j], x[j], acc);
      tmp[i] = acc;
    }
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < n; ++j) {
      float acc = 0.0f;
      for (int64_t i = 0; i < m; ++i) acc = fmaf(A[i * n + j], tmp[i], acc);
      y[j] = acc;
    }
    return 0;
  }
  double* td = (double*)malloc(sizeof(double) * (size_t)(m > 0 ? m : 1));
  if (!td) return -1;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < m; ++i) {
    double acc = 0.0;
    for (int64_t j = 0; j < n; ++j) acc += (double)A[i * n + j] * (double)x[j];
    td[i] = acc;
    tmp[i] = (float)acc;
  }
#pragma omp parallel for schedule(static)
  for (int64_t j = 0; j < n; ++j) {
    double acc = 0.0;
    for (int64_t i = 0; i < m; ++i) acc += (double)A[i * n + j] * td[i];
    y[j] = (float)acc;
  }
  free(td);
  return 0;
}

/* ---------------------------------------------------------------- BICG
 * PolyBench/GPU bicg (Table 2; Table 3), A is nx x ny:
 *   kernel 1 (column per thread):  s[j] += r[i] * A[i*ny + j]
 *   kernel 2 (row per thread):     q[i] += A[i*ny + j] * p[j]            */
int orc_bicg(int mode, const float* A, const float* p, const float* r, float* q, float* s,
             int64_t nx, int64_t ny) {
#pragma omp parallel for schedule(static)
  for (int64_t j = 0; j < ny; ++j) {
    if (mode == ORC_SEQ_FMAF) {
      float acc = 0.0f;
      for (int64_t i = 0; i < nx; ++i) acc = fmaf(r[i], A[i * ny + j], acc);
      s[j] = acc;
    } else {
      double acc = 0.0;
      for (int64_t i = 0; i < nx; ++i) acc += (double)r[i] * (double)A[i * ny + j];
      s[j] = (float)acc;
    }
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < nx; ++i) {
    if (mode == ORC_SEQ_FMAF) {
      float acc = 0.0f;
      for (int64_t j = 0; j < ny; ++j) acc = fmaf(A[i * ny + j], p[j], acc);
      q[i] = acc;
    } else {
      double acc = 0.0;
      for (int64_t j = 0; j < ny; ++j) acc += (double)A[i * ny + j] * (double)p[j];
      q[i] = (float)acc;
    }
  }
  return 0;
}

/* ---------------------------------------------------------------- MVT
 * PolyBench/GPU mvt (Table 2; Table 3), a is n x n, x1 and x2
 * are in/out (textbook MVT: x1 = x1 + A y1, x2 = x2 + A^T y2):
 *   kernel 1 (row per thread):     x1[i] += a[i*n + j] * y1[j]
 *   kernel 2 (column per thread):  x2[i] += a[j*n + i] * y2[j]           */
int orc_mvt(int mode, const float* a, const float* y1, const float* y2, float* x1, float* x2, int64_t n) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    if (mode == ORC_SEQ_FMAF) {
      float acc1 = x1[i], acc2 = x2[i];
      for (int64_t j = 0; j < n; ++j) acc1 = fmaf(a[i * n + j], y1[j], acc1);
      for (int64_t j = 0; j < n; ++j) acc2 = fmaf(a[j * n + i], y2[j], acc2);
      x1[i] = acc1;
      x2[i] = acc2;
    } else {
      double acc1 = x1[i], acc2 = x2[i];
      for (int64_t j = 0; j < n; ++j) acc1 += (double)a[i * n + j] * (double)y1[j];
      for (int64_t j = 0; j < n; ++j) acc2 += (double)a[j * n + i] * (double)y2[j];
      x1[i] = (float)acc1;
      x2[i] = (float)acc2;
    }
  }
  return 0;
}

/* ---------------------------------------------------------------- GESUMMV
 * PolyBench/GPU gesummv (Table 2 P:76 "scalar, vector, matrix
 * multiplication"; Table 3), A and B are n x n:
 *   for j: tmp[i] += A[i*n + j] * x[j];  yb[i] += B[i*n + j] * x[j];
 *   y[i] = alpha * tmp[i] + beta * yb[i]      (fused as fmaf(alpha, tmp, beta*yb))
 * tmp and y are outputs starting from 0.                                  */
int orc_gesummv(int mode, const float* A, const float* B, const float* x, float* y, float* tmp,
                int64_t n, float alpha, float beta) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    if (mode == ORC_SEQ_FMAF) {
      float t = 0.0f, yb = 0.0f;
      for (int64_t j = 0; j < n; ++j) {
        t = fmaf(A[i * n + j], x[j], t);
        yb = fmaf(B[i * n + j], x[j], yb);
      }
      tmp[i] = t;
      y[i] = fmaf(alpha, t, beta * yb);
    } else {
      double t = 0.0, yb = 0.0;
      for (int64_t j = 0; j < n; ++j) {
        t += (double)A[i * n + j] * (double)x[j];
        yb += (double)B[i * n + j] * (double)x[j];
      }
      tmp[i] = (float)t;
      y[i] = (float)((double)alpha * t + (double)beta * yb);
    }
  }
  return 0;
}

/* ---------------------------------------------------------------- three-matrix row loop
 * y[i] = (sum_j A[i][j] x[j] + sum_j B[i][j] x[j]) + sum_j C[i][j] x[j]: the
 * row loop with three memory-divergent streams per thread (not a PolyBench
 * kernel; the decision-rule studies' vehicle, DESIGN reading R29). Each sum
 * is its own fmaf chain in j order, as GESUMMV's two are (P:110-131 row form). */
int orc_rows3(int mode, const float* A, const float* B, const float* C, const float* x, float* y, int64_t m,
              int64_t n) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < m; ++i) {
    if (mode == ORC_SEQ_FMAF) {
      float a = 0.0f, b = 0.0f, c = 0.0f;
      for (int64_t j = 0; j < n; ++j) {
        a = fmaf(A[i * n + j], x[j], a);
        b = fmaf(B[i * n + j], x[j], b);
        c = fmaf(C[i * n + j], x[j], c);
      }
      y[i] = (a + b) + c;
    } else {
      double a = 0.0, b = 0.0, c = 0.0;
      for (int64_t j = 0; j < n; ++j) {
        a += (double)A[i * n + j] * (double)x[j];
        b += (double)B[i * n + j] * (double)x[j];
        c += (double)C[i * n + j] * (double)x[j];
      }
      y[i] = (float)((a + b) + c);
    }
  }
  return 0;
}

/* ---------------------------------------------------------------- SYRK
 * PolyBench/GPU syrk (Table 2; CI group), A is n x m, C is n x n in/out,
 * full square (no triangle), 2-D thread block over (i, j):
 *   c[i*n + j] *= beta;  for k: c[i*n + j] += alpha * a[i*m + k] * a[j*m + k]
 * The product alpha*a_ik is rounded first (left to right), then fused:
 *   c = fmaf(alpha * a_ik, a_jk, c).                                      */
int orc_syrk(int mode, const float* A, float* C, int64_t n, int64_t m, float alpha, float beta) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    for (int64_t j = 0; j < n; ++j) {
      if (mode == ORC_SEQ_FMAF) {
        float c = C[i * n + j] * beta;
        for (int64_t k = 0; k < m; ++k) c = fmaf(alpha * A[i * m + k], A[j * m + k], c);
        C[i * n + j] = c;
      } else {
        double c = (double)C[i * n + j] * (double)beta;
        for (int64_t k = 0; k < m; ++k) c += (double)alpha * (double)A[i * m + k] * (double)A[j * m + k];
        C[i * n + j] = (float)c;
      }
    }
  }
  return 0;
}

/* The same SYRK loop nest restricted to the output rows rows[0..nrows):
 * out[r][j] for the r-th listed row (full-size sampled checks). */
int orc_syrk_rows(int mode, const float* A, const float* C, int64_t n, int64_t m, float alpha, float beta,
                  const int64_t* rows, int64_t nrows, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t q = 0; q < nrows * n; ++q) {
    const int64_t i = rows[q / n], j = q % n;
    if (mode == ORC_SEQ_FMAF) {
      float c = C[i * n + j] * beta;
      for (int64_t k = 0; k < m; ++k) c = fmaf(alpha * A[i * m + k], A[j * m + k], c);
      out[q] = c;
    } else {
      double c = (double)C[i * n + j] * (double)beta;
      for (int64_t k = 0; k < m; ++k) c += (double)alpha * (double)A[i * m + k] * (double)A[j * m + k];
      out[q] = (float)c;
    }
  }
  return 0;
}

/* ---------------------------------------------------------------- SYR2K
 * PolyBench/GPU syr2k (Table 2; Table 3, the paper's 2-D CS
 * kernel), A and B are n x m, C is n x n in/out, full square:
 *   c[i][j] *= beta;
 *   for k: c[i][j] += alpha*a[i][k]*b[j][k] + alpha*b[i][k]*a[j][k]
 * The evaluation order of the right-hand side is fixed (R20):
 *   p = alpha*a_ik (rounded), q = alpha*b_ik (rounded),
 *   s = fmaf(p, b_jk, q*a_jk (rounded)),  c = c + s (rounded).          */
static float orc_syr2k_elem(int mode, const float* A, const float* B, const float* C, int64_t n, int64_t m,
                            float alpha, float beta, int64_t i, int64_t j) {
  if (mode == ORC_SEQ_FMAF) {
    float c = C[i * n + j] * beta;
    for (int64_t k = 0; k < m; ++k) {
      const float p = alpha * A[i * m + k];
      const float q = alpha * B[i * m + k];
      const float t = q * A[j * m + k];
      const float s = fmaf(p, B[j * m + k], t);
      c = c + s;
    }
    return c;
  }
  double c = (double)C[i * n + j] * (double)beta;
  for (int64_t k = 0; k < m; ++k)
    c += (double)alpha * (double)A[i * m + k] * (double)B[j * m + k] +
         (double)alpha * (double)B[i * m + k] * (double)A[j * m + k];
  return (float)c;
}

int orc_syr2k(int mode, const float* A, const float* B, float* C, int64_t n, int64_t m, float alpha, float beta) {
  float* out = (float*)malloc(sizeof(float) * (size_t)(n > 0 ? n * n : 1));
  if (!out) return -1;
#pragma omp parallel for schedule(static)
  for (int64_t q = 0; q < n * n; ++q) out[q] = orc_syr2k_elem(mode, A, B, C, n, m, alpha, beta, q / n, q % n);
  memcpy(C, out, sizeof(float) * (size_t)(n * n));
  free(out);
  return 0;
}

int orc_syr2k_rows(int mode, const float* A, const float* B, const float* C, int64_t n, int64_t m, float alpha,
                   float beta, const int64_t* rows, int64_t nrows, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t q = 0; q < nrows * n; ++q) out[q] = orc_syr2k_elem(mode, A, B, C, n, m, alpha, beta, rows[q / n], q % n);
  return 0;
}

/* ---------------------------------------------------------------- GEMM
 * PolyBench/GPU gemm (Table 2 CI group; the cache-insensitive
 * negative control of SURVEY 8(f) f3 / P:397). A is ni x nk, B nk x nj,
 * C ni x nj in/out:
 *   c[i][j] *= beta;  for k: c[i][j] += alpha * a[i][k] * b[k][j]
 * evaluated as c = fmaf(alpha * a_ik (rounded), b_kj, c), k ascending.   */
int orc_gemm(int mode, const float* A, const float* B, float* C, int64_t ni, int64_t nj, int64_t nk, float alpha,
             float beta) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < ni; ++i) {
    for (int64_t j = 0; j < nj; ++j) {
      if (mode == ORC_SEQ_FMAF) {
        float c = C[i * nj + j] * beta;
        for (int64_t k = 0; k < nk; ++k) c = fmaf(alpha * A[i * nk + k], B[k * nj + j], c);
        C[i * nj + j] = c;
      } else {
        double c = (double)C[i * nj + j] * (double)beta;
        for (int64_t k = 0; k < nk; ++k) c += (double)alpha * (double)A[i * nk + k] * (double)B[k * nj + j];
        C[i * nj + j] = (float)c;
      }
    }
  }
  return 0;
}

/* ---------------------------------------------------------------- CORR
 * PolyBench/GPU correlation (Table 2; Table 3; the give-up case
 * of P:244 and P:395). data is n x m (rows = observations, columns =
 * variables), centred and scaled in place; per column, i ascending:
 *   mean[j] = (sum_i data[i][j]) / fn
 *   std[j]  = sqrtf((sum_i fmaf(d, d, .), d = data[i][j] - mean[j]) / fn),
 *             std[j] = 1 if std[j] <= eps
 *   data[i][j] = (data[i][j] - mean[j]) / (sqrtf(fn) * std[j])
 *   symmat[j1][j1] = 1;  for j2 > j1: s = 0; for i: s = fmaf(data[i][j1], data[i][j2], s);
 *                        symmat[j1][j2] = symmat[j2][j1] = s
 * with fn = (float)n and eps = 0.005f (R22). Mode ORC_SEQ_F64
 * runs the same steps in double (rounded to float at the end of each). */
int orc_corr(int mode, float* data, int64_t n, int64_t m, float* mean, float* stdv, float* symmat) {
  const float fn = (float)n, eps = 0.005f;
#pragma omp parallel for schedule(static)
  for (int64_t j = 0; j < m; ++j) {
    if (mode == ORC_SEQ_FMAF) {
      float mu = 0.0f;
      for (int64_t i = 0; i < n; ++i) mu = mu + data[i * m + j];
      mu = mu / fn;
      float sd = 0.0f;
      for (int64_t i = 0; i < n; ++i) {
        const float d = data[i * m + j] - mu;
        sd = fmaf(d, d, sd);
      }
      sd = sqrtf(sd / fn);
      if (sd <= eps) sd = 1.0f;
      const float scale = sqrtf(fn) * sd;
      for (int64_t i = 0; i < n; ++i) data[i * m + j] = (data[i * m + j] - mu) / scale;
      mean[j] = mu;
      stdv[j] = sd;
    } else {
      double mu = 0.0;
      for (int64_t i = 0; i < n; ++i) mu += data[i * m + j];
      mu /= (double)n;
      double sd = 0.0;
      for (int64_t i = 0; i < n; ++i) sd += ((double)data[i * m + j] - mu) * ((double)data[i * m + j] - mu);
      sd = sqrt(sd / (double)n);
      if (sd <= (double)eps) sd = 1.0;
      for (int64_t i = 0; i < n; ++i) data[i * m + j] = (float)(((double)data[i * m + j] - mu) / (sqrt((double)n) * sd));
      mean[j] = (float)mu;
      stdv[j] = (float)sd;
    }
  }
#pragma omp parallel for schedule(dynamic, 4)
  for (int64_t j1 = 0; j1 < m; ++j1) {
    symmat[j1 * m + j1] = 1.0f;
    for (int64_t j2 = j1 + 1; j2 < m; ++j2) {
      float s;
      if (mode == ORC_SEQ_FMAF) {
        s = 0.0f;
        for (int64_t i = 0; i < n; ++i) s = fmaf(data[i * m + j1], data[i * m + j2], s);
      } else {
        double d = 0.0;
        for (int64_t i = 0; i < n; ++i) d += (double)data[i * m + j1] * (double)data[i * m + j2];
        s = (float)d;
      }
      symmat[j1 * m + j2] = s;
      symmat[j2 * m + j1] = s;
    }
  }
  return 0;
}

/* ---------------------------------------------------------------- KMEANS assign
 * Rodinia kmeans (Table 2; Table 3), assignment step
 * (kmeansPoint), features stored feature-major: feat[f*ld + p].
 *   index = -1; min = FLT_MAX;
 *   for c < k: d = 0; for f < nf: diff = feat[f*ld+p] - clusters[c*nf+f];
 *                                 d = fmaf(diff, diff, d);
 *              if (d < min) { min = d; index = c; }      (strict <: lowest c wins ties)
 * Membership decisions are taken in fp32 with this exact order in both modes
 * (an integer decided by floating point is decided in the kernel's precision,
 * DESIGN.md reading R16); mode ORC_SEQ_F64 also writes the fp64 distance
 * margin (second best - best) so tests can flag near-ties.               */
int orc_kmeans_assign(int mode, const float* feat, int64_t ld, int64_t npoints, int32_t nf,
                      const float* clusters, int32_t k, int32_t* membership, float* margin) {
#pragma omp parallel for schedule(static)
  for (int64_t p = 0; p < npoints; ++p) {
    int32_t index = -1;
    float min_dist = FLT_MAX;
    double best = INFINITY, second = INFINITY;
    for (int32_t c = 0; c < k; ++c) {
      float d = 0.0f;
      double dd = 0.0;
      for (int32_t f = 0; f < nf; ++f) {
        float diff = feat[(int64_t)f * ld + p] - clusters[(int64_t)c * nf + f];
        d = fmaf(diff, diff, d);
        if (mode == ORC_SEQ_F64) {
          double dx = (double)feat[(int64_t)f * ld + p] - (double)clusters[(int64_t)c * nf + f];
          dd += dx * dx;
        }
      }
      if (d < min_dist) {
        min_dist = d;
        index = c;
      }
      if (mode == ORC_SEQ_F64) {
        if (dd < best) { second = best; best = dd; }
        else if (dd < second) second = dd;
      }
    }
    membership[p] = index;
    if (margin) margin[p] = (mode == ORC_SEQ_F64) ? (float)(second - best) : 0.0f;
  }
  return 0;
}

/* ---------------------------------------------------------------- hashed ATAX
 * Same ATAX loop nest with A generated on the fly, A[i][j] = value(seedA,
 * i*n + j, amode) (the seeded_inputs recipe), for the full-size sampled
 * parity checks where A (4 GiB) is never materialised on the host:
 *   tmp_all[i] for every row (needed by kernel 2), then y at cols[0..ncols). */
int orc_atax_hashed(int mode, uint32_t seedA, int amode, const float* x, int64_t m, int64_t n,
                    float* tmp_all, const int64_t* cols, int64_t ncols, float* y_cols) {
  double* td = (double*)malloc(sizeof(double) * (size_t)(m > 0 ? m : 1));
  if (!td) return -1;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < m; ++i) {
    float acc = 0.0f;
    double accd = 0.0;
    for (int64_t j = 0; j < n; ++j) {
      float a = orc_value(seedA, (uint64_t)(i * n + j), amode);
      if (mode == ORC_SEQ_FMAF) acc = fmaf(a, x[j], acc);
      else accd += (double)a * (double)x[j];
    }
    tmp_all[i] = (mode == ORC_SEQ_FMAF) ? acc : (float)accd;
    td[i] = (mode == ORC_SEQ_FMAF) ? (double)acc : accd;
  }
#pragma omp parallel for schedule(static)
  for (int64_t c = 0; c < ncols; ++c) {
    int64_t j = cols[c];
    float acc = 0.0f;
    double accd = 0.0;
    for (int64_t i = 0; i < m; ++i) {
      float a = orc_value(seedA, (uint64_t)(i * n + j), amode);
      if (mode == ORC_SEQ_FMAF) acc = fmaf(a, tmp_all[i], acc);
      else accd += (double)a * td[i];
    }
    y_cols[c] = (mode == ORC_SEQ_FMAF) ? acc : (float)accd;
  }
  free(td);
  return 0;
}

void orc_set_num_threads(int n) {
#ifdef _OPENMP
  extern void omp_set_num_threads(int);
  if (n > 0) omp_set_num_threads(n);
#else
  (void)n;
#endif
}

int orc_num_threads(void) {
#ifdef _OPENMP
  extern int omp_get_max_threads(void);
  return omp_get_max_threads();
#else
  return 1;
#endif
}
