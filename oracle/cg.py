"""Oracle of the even-odd normal operator and its CG solve -- TEST INFRASTRUCTURE ONLY.

Not in the paper: SURVEY.md §8(f)-3 ("both-parity D^dag D = -D_oe D_eo, plus CG"), the solver
step that follows the Dslash in MILC's su3_rhmd_hisq.  Definitions:

    A_p x = m^2 x - D_{p,1-p} D_{1-p,p} x        on the sites of parity p,

with D_{a,b} the oracle Dslash from parity b to target parity a (oracle.dslash).  Because D is
anti-Hermitian (pin P3), A_p = m^2 + D_{1-p,p}^dag D_{1-p,p} is Hermitian positive definite.

``cg`` is the textbook conjugate-gradient iteration (Hestenes & Stiefel 1952), written out step
by step in its usual notation, starting from x_0 = 0:

    r_0 = b, p_0 = r_0
    alpha_k = <r_k, r_k> / <p_k, A p_k>
    x_{k+1} = x_k + alpha_k p_k,  r_{k+1} = r_k - alpha_k A p_k
    beta_k  = <r_{k+1}, r_{k+1}> / <r_k, r_k>,  p_{k+1} = r_{k+1} + beta_k p_k

stopping when |r_k| <= rel_tol |b|.  Pins: tests/test_oracle_cg.py (brute-force operator,
free-field closed form).
"""
from __future__ import annotations

import numpy as np

from . import dslash, parity_mask


def normal_apply(fat, lng, x, parity, mass, nthreads=0):
    """A_p x on full-lattice arrays; x is read on parity p only, the result is 0 off parity p."""
    lt, lz, ly, lx = fat.shape[:4]
    on = (parity_mask((lx, ly, lz, lt)) == bool(parity))[..., None]
    xp = np.where(on, x, 0)
    t = dslash(fat, lng, xp, 1 - parity, nthreads)          # D_{1-p,p} x
    u = dslash(fat, lng, t, parity, nthreads)               # D_{p,1-p} D_{1-p,p} x
    return np.where(on, mass * mass * xp - u, 0)


def cg(fat, lng, b, parity, mass, rel_tol=1e-12, max_iter=10000, nthreads=0):
    """Solve A_p x = b (full-lattice arrays, b on parity p).  Returns (x, iterations)."""
    lt, lz, ly, lx = fat.shape[:4]
    on = (parity_mask((lx, ly, lz, lt)) == bool(parity))[..., None]
    b = np.where(on, b, 0)
    x = np.zeros_like(b)
    r = b.copy()
    p = r.copy()
    rr = np.vdot(r, r).real
    bb = rr
    k = 0
    while k < max_iter and rr > rel_tol * rel_tol * bb:
        ap = normal_apply(fat, lng, p, parity, mass, nthreads)
        alpha = rr / np.vdot(p, ap).real
        x = x + alpha * p
        r = r - alpha * ap
        rr_new = np.vdot(r, r).real
        beta = rr_new / rr
        p = r + beta * p
        rr = rr_new
        k += 1
    return x, k
