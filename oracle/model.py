"""Oracle for NEXT-3, the analytic wasted-GPU-time model of PAPER.md §5
(TEST INFRASTRUCTURE ONLY; same import rules as oracle/oracle.py).

Each function is the paper's equation written out:
  eq. 1  W(c)/Nt = c*o + N*f*r + N*f/(2c)                      (periodic, frequency c)
  eq. 3  c*      = sqrt(N*f / (2*o))    (printed "2α": garbled 2o, reading R18)
  eq. 5  w*      = sqrt(N*f*o/2) + N*f*r + sqrt(N*f*o/2)
  eq. 6  w_f     = w / (1 + w)          (printed "W/(1+W)")
  eq. 7  w_jit   = f*o + o_jit + N*f*r + N*f*m/2                (user-level JIT)
  eq. 8  w_tjit  = o_jit + N*f*m/2                              (transparent JIT, transient)
f is the failure rate of one GPU per second, o the checkpoint time, r the fixed
recovery time, m the minibatch time (seconds), o_jit the steady-state
overhead as a fraction.  Pinned by Table 8 (tests/golden/table8.json).
"""
import math


def waste_periodic(N, f, o, r, c):
    """eq. 1 divided by N*t: wasted GPU time per GPU per unit time at frequency c."""
    return c * o + N * f * r + N * f / (2 * c)


def c_star(N, f, o):
    """eq. 3."""
    return math.sqrt(N * f / (2 * o))


def w_star(N, f, o, r):
    """eq. 5 (eq. 1 at c = c*)."""
    return math.sqrt(N * f * o / 2) + N * f * r + math.sqrt(N * f * o / 2)


def waste_fraction(w):
    """eq. 6."""
    return w / (1 + w)


def w_user_jit(N, f, o, r, m, o_jit):
    """eq. 7 divided by N*t."""
    return f * o + o_jit + N * f * r + N * f * m / 2


def w_transparent_jit(N, f, m, o_jit):
    """eq. 8 divided by N*t."""
    return o_jit + N * f * m / 2
