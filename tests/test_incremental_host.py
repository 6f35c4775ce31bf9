"""Host logic of the incremental SCF builder (no GPU): the convergence-aware threshold schedule
("relaxed thresholds in early iterations, tightened near convergence")."""
from paper_conf_sc_han0jlacz0025_b200.incremental import tau_schedule


def test_tau_schedule_clips_and_tightens():
    tf, tl, sc = 1e-12, 1e-8, 1e-5
    assert tau_schedule(1.0, tf, tl, sc) == tl            # early: loose
    assert abs(tau_schedule(1e-5, tf, tl, sc) - 1e-10) <= 1e-24  # proportional to max|dD|
    assert tau_schedule(1e-9, tf, tl, sc) == tf           # converged: final threshold
    seq = [tau_schedule(d, tf, tl, sc) for d in (1.0, 1e-2, 1e-4, 1e-6, 1e-8, 0.0)]
    assert all(a >= b for a, b in zip(seq, seq[1:]))      # monotone in max|dD|


def test_incremental_precision_schedule():
    """Convergence-aware precision (R21): thresh_fp64_n = precision_scale *
    max|Delta D_n| -- relaxed (more TF32 work) early, tight (FP64) near convergence, None when disabled."""
    from paper_conf_sc_han0jlacz0025_b200.incremental import precision_schedule
    assert precision_schedule(1.0, None) is None and precision_schedule(0.0, 1e-3) is None
    seq = [precision_schedule(d, 1e-3) for d in (1.0, 1e-2, 1e-4, 1e-6)]
    assert all(a > b for a, b in zip(seq, seq[1:]))
    assert abs(precision_schedule(1e-6, 1e-3) - 1e-9) <= 1e-24
