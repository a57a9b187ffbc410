"""Test-side parity helpers (not part of the oracle, not part of the product).

ReLU decisions (reading R30).  σ'(Z) = 1[Z > 0] is a discrete value
that floating point decides (eq. 3).  The oracle's backward
uses its own fp64 decision `ref.Z > 0`.  The kernel's fp32 forward may decide
differently only where the exact pre-activation is within rounding of zero.
`relu_tiebreak` asserts that every disagreement lies inside the declared band
|Z_ref| <= band * max|Z_ref| and only there takes the kernel's side, by moving
the oracle's Z to +/- a denormal-sized value of the kernel's sign (a change
of at most band * max|Z_ref|, below the rounding of the kernel's forward).
Outside the band the oracle decides alone.
"""
import numpy as np

# fp32 path: the kernel's forward is accurate to ~1e-6 normwise, so 2^-16.
BAND_FP32 = 2.0 ** -16
# fast variant (bf16 SpMM operand, 1xTF32 GEMM; 2e-2 gate): 2^-6.
BAND_FAST = 2.0 ** -6

_TINY = 1e-300


def relu_tiebreak(ref, H_kernel, band=BAND_FP32):
    """ref: an oracle `Result` after `forward`; H_kernel[l-1] = the kernel's H^l
    (l = 1..L-1, full N x f_l).  Asserts every sign disagreement is in the band;
    returns (#disagreements, max |Z_ref|/max|Z_ref| over them); mutates ref.Z
    at those positions only."""
    n_dis, worst = 0, 0.0
    for l, Hk in enumerate(H_kernel, start=1):
        Z = ref.Z[l]
        assert Hk.shape == Z.shape, (l, Hk.shape, Z.shape)
        kpos = np.asarray(Hk) > 0
        dis = kpos != (Z > 0)
        if not dis.any():
            continue
        zmax = float(np.abs(Z).max())
        rel = np.abs(Z[dis]) / zmax if zmax > 0 else np.zeros(int(dis.sum()))
        out = rel > band
        assert not out.any(), (
            f"layer {l}: {int(out.sum())} ReLU decisions differ outside the band "
            f"(|Z_ref|/max up to {rel.max():.3e} > {band:.3e})")
        n_dis += int(dis.sum())
        worst = max(worst, float(rel.max()))
        Zc = Z.copy()
        Zc[dis] = np.where(kpos[dis], _TINY, -_TINY)
        ref.Z[l] = Zc
    return n_dis, worst
