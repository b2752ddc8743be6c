#!/usr/bin/env python
"""Fit the odd polynomial used by the GPU's quarter-turn arctangent (csrc/device_math.cuh):

    tau(t) = (2/pi) atan(t) ~= t * P(t^2),   |t| <= tan(pi/8)

P is the Chebyshev interpolant of (2/pi) atan(sqrt(s))/sqrt(s) on s in [0, tan^2(pi/8)]
(truncated to K terms: near-minimax), computed and converted to the monomial basis in x87
extended precision.  A kernel constant table, not test data.  Prints the C table and the
max relative error (long double evaluation of the fp64-rounded coefficients).
"""
import numpy as np

L = np.longdouble
K = int(__import__("sys").argv[1]) if len(__import__("sys").argv) > 1 else 12
PI = np.arccos(L(-1))
tmax = np.tan(PI / 8)
smax = tmax * tmax
N = 64
j = np.arange(N, dtype=L)
xk = np.cos(PI * (j + L(0.5)) / N)             # Chebyshev nodes in [-1, 1]
sk = (xk + 1) * smax / 2
tk = np.sqrt(sk)
fk = (2 / PI) * np.arctan(tk) / tk
# Chebyshev coefficients a_m = 2/N sum f_k T_m(x_k)
a = np.array([(2 / L(N)) * np.sum(fk * np.cos(L(m) * PI * (j + L(0.5)) / N)) for m in range(K)])
a[0] /= 2
# convert sum a_m T_m(x), x = 2 s / smax - 1, to monomials in s (long double polynomial algebra)
def pmul(p, q):
    r = np.zeros(len(p) + len(q) - 1, dtype=L)
    for i, pi in enumerate(p):
        r[i:i + len(q)] += pi * q
    return r
x_of_s = np.array([L(-1), 2 / smax], dtype=L)
T = [np.array([L(1)]), x_of_s]
for m in range(2, K):
    T.append(np.pad(2 * pmul(x_of_s, T[-1]), (0, 0)) - np.pad(T[-2], (0, 2)))
coef = np.zeros(K, dtype=L)
for m in range(K):
    coef[:len(T[m])] += a[m] * T[m][:K]
c64 = coef.astype(np.float64)
tt = np.linspace(L(0), tmax, 400001)[1:]
ss = tt * tt
p = np.zeros_like(ss)
for c in c64[::-1].astype(L):
    p = p * ss + c
rel = np.max(np.abs(tt * p - (2 / PI) * np.arctan(tt)) / ((2 / PI) * np.arctan(tt)))
print(f"// K = {K}: max relative error of t*P(t^2) vs (2/pi)atan(t) on (0, tan(pi/8)]: {float(rel):.3e}")
print("__constant__ double kAtanQ[%d] = {" % K)
for c in c64:
    print(f"    {float(c).hex()},  // {float(c):.17g}")
print("};")
