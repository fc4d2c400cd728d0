/* CPU pin for the quotient of XS_SEARCH_S (lookup_staged.cu quotient_markstein):
 * f = RN(q0 + r*y), q0 = RN(a*y), r = fma(-d, q0, a), y = RN(1/d) must equal the IEEE
 * quotient RN(a/d) -- Markstein's theorem.  Inputs are drawn the way the lookup meets them:
 * E, q are LCG doubles (multiples of 2^-63 in [0, 1)), a = RN(E_hi - q), d = RN(E_hi - E_lo),
 * plus adversarial divisors (all-ones mantissas, powers of two, near-equal energies).
 * Built with -ffp-contract=off so every operation above is rounded exactly once.
 * usage: markstein_check N SEED  -> prints "cases mismatches" */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

static uint64_t st;
static uint64_t next(void) { st = st * 6364136223846793005ull + 1442695040888963407ull; return st; }
static double draw(void) { return (double)(next() >> 1) * 0x1p-63; } /* [0, 1), multiple of 2^-63 */

static int check(double a, double d)
{
    const double y = 1.0 / d;
    const double q0 = a * y;
    const double r = fma(-d, q0, a);
    const double f = fma(r, y, q0);
    const double ref = a / d;
    return f != ref && !(f != f && ref != ref);
}

int main(int argc, char **argv)
{
    const long n = argc > 1 ? atol(argv[1]) : 1000000;
    st = argc > 2 ? strtoull(argv[2], 0, 10) : 1;
    long bad = 0, cases = 0;
    for (long i = 0; i < n; i++) {
        double lo = draw(), hi = draw();
        if (lo == hi) continue;
        if (lo > hi) { double t = lo; lo = hi; hi = t; }
        const int mode = (int)(next() >> 61);
        double q;
        if (mode == 0) q = lo + (hi - lo) * draw();          /* inside the interval */
        else if (mode == 1) q = draw();                       /* anywhere (extrapolation) */
        else if (mode == 2) q = lo;                           /* at the lower point (f = 1) */
        else if (mode == 3) q = hi;                           /* at the upper point (f = 0) */
        else if (mode == 4) {                                 /* near-equal energies */
            hi = nextafter(lo, 2.0);
            for (int k = (int)(next() >> 60); k > 0; k--) hi = nextafter(hi, 2.0);
            q = lo + (hi - lo) * draw();
        } else if (mode == 5) {                               /* all-ones-mantissa divisor */
            const int e = -(int)(next() >> 59) - 1;
            hi = lo + ldexp(0x1.fffffffffffffp0, e);
            q = draw();
        } else if (mode == 6) {                               /* power-of-two divisor */
            hi = lo + ldexp(1.0, -(int)(next() >> 59) - 1);
            q = draw();
        } else q = hi - (hi - lo) * 0x1p-40 * draw();           /* f near 0 */
        const double d = hi - lo, a = hi - q;
        if (d == 0.0 || !isfinite(d)) continue;
        bad += check(a, d);
        cases++;
    }
    printf("%ld %ld\n", cases, bad);
    return 0;
}
