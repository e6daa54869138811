"""Physics validation through the whole GPU path (the paper's Sec. V-A):
history ring -> retarded potentials -> fields (R-15b) -> forces on particles (rp_particle_forces,
the push's gather), for a Gaussian bunch (sigma = 50 um, Q = 1) in steady-state circular motion
on the LCLS orbit (R0 = 25.13 m, gamma = 1e4), tools/csr_validation.py:

* Fig. 2: longitudinal AND transverse forces on test particles on the bunch axis and 1 sigma off
  it, against the exact steady-state solution of the same sheet bunch (1-D quadrature of the
  theta-closed form of Eq. 1, no grid) and the longitudinal one also against the 1D line-charge
  CSR formula (Derbenev et al. 1995; Saldin et al. 1997).  Measured at 129^2 (r02): 0.37 % /
  0.16 % (axis F_s / F_n) and 0.36 % / 0.14 % (off axis) of the peak; exact sheet vs line 0.06 %.
* Fig. 3: mean-square error of the particle forces against the noise-free expected deposit vs N
  -- "scales as 1/N"; measured slope -1.03 (F_s), -0.97 (F_n) over 1e4..1e7.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def test_steady_state_forces_match_the_exact_solution():
    from tools.csr_validation import validate_forces
    rec = validate_forces(n=129, offsets=np.linspace(-3.0, 3.0, 13))
    for key in ("max_rel_dev_Fs_axis", "max_rel_dev_Fn_axis", "max_rel_dev_Fs_v+1sigma",
                "max_rel_dev_Fn_v+1sigma"):
        assert rec[key] <= 0.01, (key, rec[key])
    # the exact sheet solution is the 1D line-charge CSR field on the axis (independent formula)
    assert rec["max_rel_dev_exact_sheet_vs_1d_line"] <= 0.002
    assert rec["max_rel_dev_Fs_axis_vs_1d_line"] <= 0.01
    # the CSR signature: decelerating core, accelerating head; inward transverse force
    fs = np.array(rec["gpu_Fs_axis"])
    offs = np.array(rec["s_over_sigma"])
    assert fs[np.argmin(np.abs(offs + 0.5))] < 0 < fs[np.argmin(np.abs(offs - 2.0))]
    assert np.all(np.array(rec["gpu_Fn_axis"]) < 0)


def test_force_mean_square_error_scales_as_one_over_n():
    from tools.csr_validation import mse_study
    out = mse_study(ns=(10_000, 100_000, 1_000_000))
    assert abs(out["slope_Fs"] + 1.0) <= 0.15, out["slope_Fs"]
    assert abs(out["slope_Fn"] + 1.0) <= 0.15, out["slope_Fn"]
    # the noise-free reference itself sits on the exact solution at the particles
    assert out["ref_vs_exact_Fs_max_over_peak"] <= 0.02
