"""Incremental direct-SCF J/K with density-weighted screening and a convergence-aware threshold
(S3.2.3 "Convergence-aware scheduling": density-weighted Schwarz
tiers at the integral level, "relaxed thresholds in early iterations, tightened near convergence"
at the iteration level).

J and K are linear in D, so over an SCF run
    J[D_n] = J[D_{n-1}] + J[D_n - D_{n-1}]        (same for K)
and the update is built with mako_build_jk_ex(MAKO_JK_DENSITY_SCREEN) on Delta D: a quartet is
skipped when Q_ab Q_cd max|Delta D| (over its six shell blocks) < tau_n, so the work shrinks with
Delta D as the SCF converges.  The screening error of one build is bounded per dropped quartet by
2 tau_n (include/mako.h); it accumulates over incremental builds, so the builder rebuilds from the
full density (a) every `rebuild_every` builds, (b) when the threshold reaches tau_final (the
converged Fock matrix then carries only tau_final-level screening error) and (c) when it has
tightened by more than a factor `tighten` since the last full build.  The schedule (reading R18):
    tau_n = clip(tau_scale * max|Delta D_n|, tau_final, tau_loose)
i.e. the neglected Fock contributions stay a fixed factor below the current density change.
With `precision_scale` set, every build is also stage-aware mixed precision (mako_build_jk_mixed,
SURVEY S8.f row 1; "relaxed precision thresholds during early iterations - favoring
quantized kernels - and gradually tightening them as convergence nears"): quartets whose
contribution bound Q_ab Q_cd max|D_build| is below thresh_fp64_n = precision_scale * max|Delta D_n|
run the TF32 tier, so the reduced-precision share shrinks as the SCF converges (R21).  All
device work runs in libmako's kernels: Delta D and max|Delta D| come from mako_density_delta, the
update is accumulated into J/K by mako_build_jk_ex / _mixed with MAKO_JK_ACCUMULATE.
"""
import torch

from .mako import build_jk, density_delta


def tau_schedule(dmax, tau_final, tau_loose, tau_scale):
    """Convergence-aware threshold for a build whose density change has max-norm `dmax`."""
    t = tau_scale * float(dmax)
    return min(tau_loose, max(tau_final, t))


def precision_schedule(dmax, precision_scale):
    """thresh_fp64 of a build whose density change has max-norm `dmax` (None = FP64 only): quartets
    whose contribution bound Q_ab Q_cd max|D_build| is below it run the TF32 tier (R21)."""
    if precision_scale is None or not dmax > 0:
        return None
    return float(precision_scale) * float(dmax)


class IncrementalJK:
    """Callable J/K builder for an SCF loop: ``J, K = inc(D)`` with D a device (or numpy) density.

    Keeps D_{n-1}, J_{n-1}, K_{n-1} on the device.  `history` records, per call, whether it was a
    full or an incremental build, the threshold used, max|Delta D| and the device milliseconds."""

    def __init__(self, pairs, tau_final=None, tau_loose=1e-10, tau_scale=1e-7, rebuild_every=10, tighten=1e-3,
                 device=None, precision_scale=None):
        self.pairs = pairs
        self.tau_final = float(pairs.tau if tau_final is None else tau_final)
        self.tau_loose = max(float(tau_loose), self.tau_final)
        self.tau_scale = float(tau_scale)
        self.rebuild_every = int(rebuild_every)
        self.tighten = float(tighten)
        self.precision_scale = None if precision_scale is None else float(precision_scale)
        self.device = device or torch.device("cuda")
        self.D = self.J = self.K = None
        self.dD = None
        self.since_full = 0
        self.tau_full = None
        self.history = []

    def reset(self):
        self.D = self.J = self.K = None

    def __call__(self, D, return_numpy=True):
        numpy_in = not isinstance(D, torch.Tensor)
        Dt = torch.as_tensor(D, dtype=torch.float64, device=self.device).contiguous()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record()
        if self.D is None:
            self.dD = torch.empty_like(Dt)
            zero = torch.zeros_like(Dt)
            _, dmax = density_delta(self.pairs, Dt, zero, self.dD)  # max|D| through the library
            del zero
        else:
            _, dmax = density_delta(self.pairs, Dt, self.D, self.dD)
        tau = tau_schedule(dmax, self.tau_final, self.tau_loose, self.tau_scale)
        full = (self.D is None or self.since_full >= self.rebuild_every or
                (tau < self.tau_full and (tau <= self.tau_final or tau < self.tighten * self.tau_full)))
        t64 = precision_schedule(dmax, self.precision_scale)
        if full:
            if self.J is None:
                self.J, self.K = torch.empty_like(Dt), torch.empty_like(Dt)
            build_jk(self.pairs, Dt, thresh=tau, J=self.J, K=self.K, density_screen=True, thresh_fp64=t64)
            self.since_full = 0
            self.tau_full = tau
        else:  # J += J[dD], K += K[dD] inside the library
            build_jk(self.pairs, self.dD, thresh=tau, J=self.J, K=self.K, density_screen=True, thresh_fp64=t64,
                     accumulate=True)
            self.since_full += 1
        if self.D is None:
            self.D = torch.empty_like(Dt)
        self.D.copy_(Dt)
        ev1.record()
        torch.cuda.synchronize()
        self.history.append({"full": full, "tau": tau, "dmax": dmax, "thresh_fp64": t64, "ms": ev0.elapsed_time(ev1)})
        if numpy_in and return_numpy:
            return self.J.cpu().numpy(), self.K.cpu().numpy()
        return self.J, self.K
