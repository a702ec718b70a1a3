// Host-side substitution models and their eigensystems (C++, fp64).
//
// The library's K1 kernel needs Q = V diag(lambda) V^-1 (rrl.h,
// rrl_set_eigen_decomposition).  The paper's models are "time-reversible"
// (§V-A); which ones is not stated, readings A2/A13 fix
// JC69, HKY, GTR and GY94.  Reversibility makes S = Pi^1/2 Q Pi^-1/2
// symmetric, so a cyclic Jacobi sweep gives S = U diag(lambda) U^T and
// V = Pi^-1/2 U, V^-1 = U^T Pi^1/2 exactly inverse to each other.
#include <cmath>
#include <cstring>
#include <string>
#include <vector>

#include "rrl.h"
#include "rrl_internal.h"

namespace {

// Standard genetic code, codons in ACGT-lexicographic order (first base
// slowest): AAA AAC AAG AAT ACA ... TTT.  '*' = stop.
const char kCodeACGT[] = "KNKNTTTTRSRSIIMIQHQHPPPPRRRRLLLLEDEDAAAAGGGGVVVV*Y*YSSSS*CWCLFLF";

bool transition(int x, int y) {  // A=0 C=1 G=2 T=3 ; A<->G, C<->T
  return (x == 0 && y == 2) || (x == 2 && y == 0) || (x == 1 && y == 3) || (x == 3 && y == 1);
}

void jacobi_eigen(int s, std::vector<double> &A, std::vector<double> &U, std::vector<double> &lam) {
  U.assign((size_t)s * s, 0.0);
  for (int i = 0; i < s; ++i) U[(size_t)i * s + i] = 1.0;
  for (int sweep = 0; sweep < 100; ++sweep) {
    double off = 0.0, diag = 0.0;
    for (int i = 0; i < s; ++i)
      for (int j = 0; j < s; ++j) {
        const double v = A[(size_t)i * s + j] * A[(size_t)i * s + j];
        if (i == j) diag += v; else off += v;
      }
    if (off <= 1e-32 * (diag + 1e-300)) break;
    for (int p = 0; p < s - 1; ++p) {
      for (int q = p + 1; q < s; ++q) {
        const double apq = A[(size_t)p * s + q];
        if (std::fabs(apq) < 1e-300) continue;
        const double app = A[(size_t)p * s + p], aqq = A[(size_t)q * s + q];
        const double theta = (aqq - app) / (2.0 * apq);
        const double t = (theta >= 0 ? 1.0 : -1.0) / (std::fabs(theta) + std::sqrt(theta * theta + 1.0));
        const double c = 1.0 / std::sqrt(t * t + 1.0), sn = t * c;
        for (int k = 0; k < s; ++k) {  // rotate columns p, q
          const double akp = A[(size_t)k * s + p], akq = A[(size_t)k * s + q];
          A[(size_t)k * s + p] = c * akp - sn * akq;
          A[(size_t)k * s + q] = sn * akp + c * akq;
        }
        for (int k = 0; k < s; ++k) {  // rotate rows p, q
          const double apk = A[(size_t)p * s + k], aqk = A[(size_t)q * s + k];
          A[(size_t)p * s + k] = c * apk - sn * aqk;
          A[(size_t)q * s + k] = sn * apk + c * aqk;
        }
        for (int k = 0; k < s; ++k) {
          const double ukp = U[(size_t)k * s + p], ukq = U[(size_t)k * s + q];
          U[(size_t)k * s + p] = c * ukp - sn * ukq;
          U[(size_t)k * s + q] = sn * ukp + c * ukq;
        }
      }
    }
  }
  lam.resize(s);
  for (int i = 0; i < s; ++i) lam[i] = A[(size_t)i * s + i];
}

}  // namespace

extern "C" int rrl_model_eigensystem(const char *model, int s, const double *pi,
                                     const double *params, int nparams, double *Qout,
                                     double *Vout, double *Viout, double *lamout) {
  try {
    if (!model || !pi) return rrl::fail(RRL_ERROR_GENERAL, "model/pi NULL");
    const std::string m(model);
    for (int i = 0; i < s; ++i)
      if (!(pi[i] > 0)) return rrl::fail(RRL_ERROR_GENERAL, "pi must be positive");
    std::vector<double> Q((size_t)s * s, 0.0);
    if (m == "jc69" || m == "hky" || m == "gtr") {
      if (s != 4) return rrl::fail(RRL_ERROR_NO_IMPLEMENTATION, "nucleotide models need s=4");
      double r[4][4];
      for (int i = 0; i < 4; ++i)
        for (int j = 0; j < 4; ++j) r[i][j] = 1.0;
      if (m == "hky") {
        if (nparams < 1) return rrl::fail(RRL_ERROR_GENERAL, "hky needs kappa");
        for (int i = 0; i < 4; ++i)
          for (int j = 0; j < 4; ++j) r[i][j] = transition(i, j) ? params[0] : 1.0;
      } else if (m == "gtr") {
        if (nparams < 6) return rrl::fail(RRL_ERROR_GENERAL, "gtr needs 6 exchangeabilities");
        const int pr[6][2] = {{0, 1}, {0, 2}, {0, 3}, {1, 2}, {1, 3}, {2, 3}};
        for (int k = 0; k < 6; ++k) r[pr[k][0]][pr[k][1]] = r[pr[k][1]][pr[k][0]] = params[k];
      }
      for (int i = 0; i < 4; ++i)
        for (int j = 0; j < 4; ++j)
          if (i != j) Q[i * 4 + j] = r[i][j] * (m == "jc69" ? 1.0 : pi[j]);
    } else if (m == "gy94") {
      if (s != 61) return rrl::fail(RRL_ERROR_NO_IMPLEMENTATION, "gy94 needs s=61");
      if (nparams < 2) return rrl::fail(RRL_ERROR_GENERAL, "gy94 needs kappa, omega");
      const double kappa = params[0], omega = params[1];
      int sense[61], ns = 0;
      for (int c = 0; c < 64; ++c)
        if (kCodeACGT[c] != '*') sense[ns++] = c;
      if (ns != 61) return rrl::fail(RRL_ERROR_GENERAL, "genetic code table");
      for (int i = 0; i < 61; ++i)
        for (int j = 0; j < 61; ++j) {
          if (i == j) continue;
          const int ci = sense[i], cj = sense[j];
          int diffs = 0, pos = -1;
          for (int k = 0; k < 3; ++k) {
            const int sh = 2 * (2 - k);
            if (((ci >> sh) & 3) != ((cj >> sh) & 3)) { ++diffs; pos = sh; }
          }
          if (diffs != 1) continue;
          double q = pi[j];
          if (transition((ci >> pos) & 3, (cj >> pos) & 3)) q *= kappa;
          if (kCodeACGT[ci] != kCodeACGT[cj]) q *= omega;
          Q[(size_t)i * 61 + j] = q;
        }
    } else {
      return rrl::fail(RRL_ERROR_NO_IMPLEMENTATION, "unknown model");
    }
    // diagonal and normalisation -sum_i pi_i Q_ii = 1
    double rate = 0.0;
    for (int i = 0; i < s; ++i) {
      double row = 0.0;
      for (int j = 0; j < s; ++j)
        if (j != i) row += Q[(size_t)i * s + j];
      Q[(size_t)i * s + i] = -row;
      rate += pi[i] * row;
    }
    for (auto &q : Q) q /= rate;
    if (Qout) std::memcpy(Qout, Q.data(), sizeof(double) * s * s);
    // symmetric form
    std::vector<double> sq(s), S((size_t)s * s), U, lam;
    for (int i = 0; i < s; ++i) sq[i] = std::sqrt(pi[i]);
    for (int i = 0; i < s; ++i)
      for (int j = 0; j < s; ++j) S[(size_t)i * s + j] = sq[i] * Q[(size_t)i * s + j] / sq[j];
    for (int i = 0; i < s; ++i)  // symmetrise round-off
      for (int j = i + 1; j < s; ++j) {
        const double avg = 0.5 * (S[(size_t)i * s + j] + S[(size_t)j * s + i]);
        S[(size_t)i * s + j] = S[(size_t)j * s + i] = avg;
      }
    jacobi_eigen(s, S, U, lam);
    for (int i = 0; i < s; ++i)
      for (int k = 0; k < s; ++k) {
        if (Vout) Vout[(size_t)i * s + k] = U[(size_t)i * s + k] / sq[i];
        if (Viout) Viout[(size_t)k * s + i] = U[(size_t)i * s + k] * sq[i];
      }
    if (lamout) std::memcpy(lamout, lam.data(), sizeof(double) * s);
    return RRL_SUCCESS;
  } catch (...) {
    return rrl::fail(RRL_ERROR_UNIDENTIFIED_EXCEPTION, "exception in rrl_model_eigensystem");
  }
}
