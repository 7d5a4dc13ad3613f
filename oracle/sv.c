/* ORACLE -- test infrastructure only. Never linked into the product library.
 *
 * Plain state-vector update loops, written straight from the paper's definition:
 *   - the state is 2^n complex128 amplitudes, index i = sum_q b_q 2^q (Eq.3-4;
 *     little-endian, "a gate on qubit 0 requires amplitudes a_x..x0 and a_x..x1");
 *   - a k-qubit gate is a 2^k x 2^k unitary; for every index whose target bits are 0
 *     the 2^k amplitudes that differ only in the target bits are multiplied by U (Eq.8,
 *     P:70-75, generalised to k=2 per P:58); a controlled gate acts only where every control
 *     bit is 1.
 *   - measurement probabilities are |a|^2 (Eq.1), summed into marginal buckets.
 * No blocking, no reordering, no pruning: every base index of the full 2^n range is visited.
 */
#include <complex.h>
#include <stdint.h>
#include <string.h>
#include <stdlib.h>

typedef double complex cplx;

/* psi: 2^n amplitudes; U: (2^t)x(2^t) row-major; row/col bit j <-> targets[j]. */
int sv_apply(cplx *psi, int n, const cplx *U, int t, const int *targets, int nc,
             const int *controls, int threads)
{
    if (t < 1 || t > 3) return 1;
    const int64_t N = (int64_t)1 << n;
    const int dim = 1 << t;
    int64_t tmask = 0, cmask = 0;
    for (int j = 0; j < t; ++j) tmask |= (int64_t)1 << targets[j];
    for (int j = 0; j < nc; ++j) cmask |= (int64_t)1 << controls[j];
    /* offset of local basis state j: sum_k j_k 2^targets[k] */
    int64_t off[8];
    for (int j = 0; j < dim; ++j) {
        off[j] = 0;
        for (int k = 0; k < t; ++k)
            if ((j >> k) & 1) off[j] |= (int64_t)1 << targets[k];
    }
#pragma omp parallel for schedule(static) num_threads(threads)
    for (int64_t i = 0; i < N; ++i) {
        if ((i & tmask) != 0) continue;          /* visit each group once, at its base  */
        if ((i & cmask) != cmask) continue;      /* controls must all be |1>            */
        cplx v[8], w[8];
        for (int j = 0; j < dim; ++j) v[j] = psi[i + off[j]];
        for (int r = 0; r < dim; ++r) {
            cplx s = 0;
            for (int c = 0; c < dim; ++c) s += U[r * dim + c] * v[c];
            w[r] = s;
        }
        for (int j = 0; j < dim; ++j) psi[i + off[j]] = w[j];
    }
    return 0;
}

/* p(y) = sum_{i : bits_Q(i) = y} |psi_i|^2, with qubits[0] <-> bit 0 of y. */
void sv_probabilities(const cplx *psi, int n, int m, const int *qubits, double *out)
{
    const int64_t N = (int64_t)1 << n;
    memset(out, 0, sizeof(double) * ((size_t)1 << m));
    for (int64_t i = 0; i < N; ++i) {
        int64_t y = 0;
        for (int j = 0; j < m; ++j) y |= ((i >> qubits[j]) & 1) << j;
        out[y] += creal(psi[i]) * creal(psi[i]) + cimag(psi[i]) * cimag(psi[i]);
    }
}

/* z[j] = 1 iff every amplitude of chunk j (2^c amplitudes, j = index >> c) is exactly 0.0
 * (the "data zero map" used to check the soundness of the pruning bitmap). */
void sv_zero_map(const cplx *psi, int n, int c, uint8_t *z)
{
    const int64_t nch = (int64_t)1 << (n - c);
    const int64_t L = (int64_t)1 << c;
    for (int64_t j = 0; j < nch; ++j) {
        uint8_t zero = 1;
        for (int64_t k = 0; k < L; ++k) {
            cplx a = psi[j * L + k];
            if (creal(a) != 0.0 || cimag(a) != 0.0) { zero = 0; break; }
        }
        z[j] = zero;
    }
}
