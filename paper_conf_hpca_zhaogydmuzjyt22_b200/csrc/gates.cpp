// Gate table of the product path (a1). Qiskit conventions including global phase, because the
// paper extends Qiskit-Aer (reading Q10 in DESIGN.md). H is Eq.5,
// CNOT P:239, "cp" P:409. Independent of the oracle's table (oracle/qasm.py).
#include <cmath>
#include <cstring>
#include <string>
#include <vector>

#include "qgpu_internal.h"

namespace qgpu {
namespace {

inline cplx C(double re, double im = 0.0) { return cplx{re, im}; }
inline cplx expi(double a) { return cplx{std::cos(a), std::sin(a)}; }
inline cplx cmul(cplx a, cplx b) { return cplx{a.re * b.re - a.im * b.im, a.re * b.im + a.im * b.re}; }
inline cplx neg(cplx a) { return cplx{-a.re, -a.im}; }

void set2(cplx* U, cplx a, cplx b, cplx c, cplx d) { U[0] = a; U[1] = b; U[2] = c; U[3] = d; }

void u3(cplx* U, double th, double ph, double la) {
  const double c = std::cos(th / 2), s = std::sin(th / 2);
  set2(U, C(c), neg(cmul(expi(la), C(s))), cmul(expi(ph), C(s)), cmul(expi(ph + la), C(c)));
}

}  // namespace

bool gate_matrix(const std::string& nm, const std::vector<double>& p, int* np, int* nq, int* nc,
                 cplx* U, bool build) {
  const double r2 = 0.70710678118654752440;  // 1/sqrt(2), correctly rounded (= M_SQRT1_2)
  struct Ar { const char* n; int np, nq, nc; };
  static const Ar table[] = {
      {"id", 0, 1, 0},   {"x", 0, 1, 0},    {"y", 0, 1, 0},    {"z", 0, 1, 0},
      {"h", 0, 1, 0},    {"s", 0, 1, 0},    {"sdg", 0, 1, 0},  {"t", 0, 1, 0},
      {"tdg", 0, 1, 0},  {"sx", 0, 1, 0},   {"sxdg", 0, 1, 0}, {"rx", 1, 1, 0},
      {"ry", 1, 1, 0},   {"rz", 1, 1, 0},   {"p", 1, 1, 0},    {"u1", 1, 1, 0},
      {"u2", 2, 1, 0},   {"u3", 3, 1, 0},   {"u", 3, 1, 0},    {"U", 3, 1, 0},
      {"cx", 0, 2, 1},   {"CX", 0, 2, 1},   {"cy", 0, 2, 1},   {"cz", 0, 2, 1},
      {"ch", 0, 2, 1},   {"cp", 1, 2, 1},   {"cu1", 1, 2, 1},  {"crx", 1, 2, 1},
      {"cry", 1, 2, 1},  {"crz", 1, 2, 1},  {"cu3", 3, 2, 1},  {"ccx", 0, 3, 2},
      {"cswap", 0, 3, 1}, {"swap", 0, 2, 0}, {"rzz", 1, 2, 0},
  };
  const Ar* a = nullptr;
  for (const Ar& e : table)
    if (nm == e.n) { a = &e; break; }
  if (!a) return false;
  *np = a->np; *nq = a->nq; *nc = a->nc;
  if (!build) return true;
  std::string b = nm;
  // controlled forms: strip the leading 'c' (or "cc") to get the target gate
  if (a->nc == 2) b = "x";
  else if (nm == "cswap") b = "swap";
  else if (a->nc == 1) b = (nm == "CX") ? "x" : nm.substr(1);
  const int nt = a->nq - a->nc;
  for (int i = 0; i < (1 << (2 * nt)); ++i) U[i] = C(0);
  if (b == "id") set2(U, C(1), C(0), C(0), C(1));
  else if (b == "x") set2(U, C(0), C(1), C(1), C(0));
  else if (b == "y") set2(U, C(0), C(0, -1), C(0, 1), C(0));
  else if (b == "z") set2(U, C(1), C(0), C(0), C(-1));
  else if (b == "h") set2(U, C(r2), C(r2), C(r2), C(-r2));
  else if (b == "s") set2(U, C(1), C(0), C(0), C(0, 1));
  else if (b == "sdg") set2(U, C(1), C(0), C(0), C(0, -1));
  else if (b == "t") set2(U, C(1), C(0), C(0), C(r2, r2));
  else if (b == "tdg") set2(U, C(1), C(0), C(0), C(r2, -r2));
  else if (b == "sx") set2(U, C(0.5, 0.5), C(0.5, -0.5), C(0.5, -0.5), C(0.5, 0.5));
  else if (b == "sxdg") set2(U, C(0.5, -0.5), C(0.5, 0.5), C(0.5, 0.5), C(0.5, -0.5));
  else if (b == "rx") {
    const double c = std::cos(p[0] / 2), s = std::sin(p[0] / 2);
    set2(U, C(c), C(0, -s), C(0, -s), C(c));
  } else if (b == "ry") {
    const double c = std::cos(p[0] / 2), s = std::sin(p[0] / 2);
    set2(U, C(c), C(-s), C(s), C(c));
  } else if (b == "rz") set2(U, expi(-p[0] / 2), C(0), C(0), expi(p[0] / 2));
  else if (b == "p" || b == "u1") set2(U, C(1), C(0), C(0), expi(p[0]));
  else if (b == "u2") u3(U, M_PI / 2, p[0], p[1]);
  else if (b == "u3" || b == "u" || b == "U") u3(U, p[0], p[1], p[2]);
  else if (b == "swap") { U[0] = C(1); U[1 * 4 + 2] = C(1); U[2 * 4 + 1] = C(1); U[15] = C(1); }
  else if (b == "rzz") {
    U[0] = expi(-p[0] / 2); U[5] = expi(p[0] / 2); U[10] = expi(p[0] / 2); U[15] = expi(-p[0] / 2);
  } else return false;
  return true;
}

bool is_diagonal(const cplx* U, int nt) {
  const int d = 1 << nt;
  for (int r = 0; r < d; ++r)
    for (int c = 0; c < d; ++c)
      if (r != c && (U[r * d + c].re != 0.0 || U[r * d + c].im != 0.0)) return false;
  return true;
}

bool is_swap_matrix(const cplx* U, int nt) {
  if (nt != 2) return false;
  static const int one[4][2] = {{0, 0}, {1, 2}, {2, 1}, {3, 3}};
  for (int r = 0; r < 4; ++r)
    for (int c = 0; c < 4; ++c) {
      bool want = false;
      for (auto& o : one) want |= (o[0] == r && o[1] == c);
      const cplx v = U[r * 4 + c];
      if (v.im != 0.0 || v.re != (want ? 1.0 : 0.0)) return false;
    }
  return true;
}

}  // namespace qgpu
