/* Exhaustive pin of oracle_nint_sqrt over every reachable squared distance
 * s in [0, 2*32767^2] (coordinates in [0, 2^15), reading R4).  Independent
 * path: walk the rounding intervals of the definition nint(sqrt(s)) = m  <=>
 * m - 1/2 <= sqrt(s) < m + 1/2  <=>  m^2 - m < s <= m^2 + m (integer s), using
 * only integer arithmetic, and compare every s against the oracle.
 * Built and run by tests/test_oracle_exhaustive.py. */
#include <stdint.h>
#include <stdio.h>
int64_t oracle_nint_sqrt(int64_t s);
int main(void)
{
    const int64_t smax = 2LL * 32767 * 32767;
    int64_t bad = 0, checked = 0;
#pragma omp parallel for schedule(dynamic, 64) reduction(+ : bad, checked)
    for (int64_t m = 0; m <= 46341; m++) {
        int64_t lo = (m == 0) ? 0 : m * m - m + 1, hi = m * m + m;
        if (hi > smax) hi = smax;
        for (int64_t s = lo; s <= hi; s++) {
            checked++;
            if (oracle_nint_sqrt(s) != m) bad++;
        }
    }
    printf("%lld %lld\n", (long long)checked, (long long)bad);
    return !(bad == 0 && checked == smax + 1);
}
