"""Window solver (sh_solve_window, C-ABI, no GPU) vs the paper's model.

Pins: homogeneous closed forms derived by hand from eq. 1b / 2b / 1d / 2d, the memory
fallback of PAPER.md:195 -- each run against both the C++ solver and the brute-force
transcription in oracle/autotune_oracle.py (the oracle's own pin) -- and agreement of the two on
random heterogeneous profiles.
"""
import math

import numpy as np
import pytest

from oracle import autotune_oracle as AO

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")


class Infeasible(Exception):
    """No window fits the memory (the C-ABI returns SH_ERR_OOM_DEVICE, the oracle None)."""


def _engine(**kw):
    try:
        return sh.solve_window(**kw)
    except sh.ShError as e:
        if e.status == sh.SH_ERR_OOM_DEVICE:
            raise Infeasible from e
        raise


def _oracle(**kw):
    r = AO.solve(**kw)
    if r is None:
        raise Infeasible
    return r


@pytest.fixture(params=["engine", "oracle"])
def solve(request):
    """Every closed-form pin below runs against BOTH the C++ solver and the brute-force oracle, so
    the oracle is pinned by hand-derived values, not only by agreement with the code it checks."""
    return {"engine": _engine, "oracle": _oracle}[request.param]


def homog(L, a, c, d, **kw):
    """t_fp = a, t_bp = 3a (recompute + 2x backward, PAPER.md:153 fn. 2), t_c2g = c, t_g2c = d."""
    return dict(t_fp=[a] * L, t_bp=[3 * a] * L, t_c2g=[c] * L, t_g2c=[d] * L, **kw)


def test_homogeneous_fp_bound_closed_form(solve):
    # soft fails (a < c + d) => w* = smallest w with w a >= c and 3 w a >= max(c, d)
    for a, c, d in [(1.0, 2.5, 1.0), (2.0, 9.0, 3.0), (1.0, 0.9, 0.2), (0.5, 3.2, 7.0)]:
        L = 40
        r = solve(**homog(L, a, c, d))
        expect = max(math.ceil(c / a), math.ceil(max(c, d) / (3 * a)))
        if a >= c + d:  # soft holds at the hard minimum too
            assert r["reason"] == 0
        else:
            assert r["reason"] == 1
        assert r["window"] == expect, (a, c, d, r)


def test_soft_constraint_met_gives_reason0_and_no_jump_to_resident(solve):
    # a >= c + d: every w meeting hard meets soft; the solver must not pick w = L
    r = solve(**homog(24, 4.0, 3.0, 0.5))
    assert r == {**r, "window": 1, "reason": 0}
    # soft unsatisfiable: still the hard minimum, not the vacuous w = L
    r = solve(**homog(24, 1.0, 1.5, 2.0))
    assert r["window"] == 2 and r["reason"] == 1


def test_memory_fallback_largest_window(solve):
    # hard needs w >= 5 but memory allows only w <= 3 -> w* = 3
    L = 20
    prof = homog(L, 1.0, 5.0, 1.0, slot_bytes=[100] * L, gstate_bytes=[50] * L, fixed_bytes=0,
                 s_avail=4 * 100 + 3 * 50)
    r = solve(**prof)
    assert r["window"] == 3 and r["reason"] == 2 and r["w_max_memory"] == 3


def test_oom_even_at_w0(solve):
    with pytest.raises(Infeasible):
        solve(**homog(4, 1, 1, 1, slot_bytes=[10] * 4, s_avail=5))


def test_resident_when_transfers_cannot_hide_and_memory_allows(solve):
    # no w < L meets the FP hard constraint (c2g exceeds the whole model's FP time), memory allows L
    L = 6
    r = solve(**homog(L, 1.0, 100.0, 1.0))
    assert r["window"] == L and r["reason"] == 1


def test_cpu_hard_pushes_window_up(solve):
    L = 10
    prof = homog(L, 1.0, 0.5, 0.5, t_opt_cpu=[10.0] * L, t_opt_gpu=[0.1] * L)
    r0 = solve(**prof)
    assert r0["window"] == 1
    r1 = solve(**prof, cpu_hard=True)
    # (L - w) * 10 <= 4 L + 0.1 w  ->  w >= (10 L - 4 L) / 10.1
    assert r1["window"] == math.ceil((10 * L - 4 * L) / 10.1)
    assert r1["cpu_total_ms"] <= r1["gpu_step_ms"]
    # utilisation target rho = 0.5: (L - w) * 10 <= 0.5 (4 L + 0.1 w)
    r2 = solve(**prof, cpu_hard=True, cpu_util_max=0.5)
    assert r2["window"] == math.ceil((10 * L - 2 * L) / 10.05)


def test_eq3_and_eq4_reports(solve):
    L = 8
    prof = homog(L, 1.0, 0.5, 0.2, t_opt_cpu=[3.0] * L, t_opt_gpu=[0.25] * L, t_async=0.01)
    r = solve(**prof)
    w = r["window"]
    # slack at k = w: (w+1)*4 + 0.25 w - 3
    assert abs(r["eq3_min_slack_ms"] - ((w + 1) * 4.0 + 0.25 * w - 3.0)) < 1e-12
    assert abs(r["eq4_lhs_ms"] - 5 * L * 0.01) < 1e-12
    assert abs(r["eq4_rhs_ms"] - 0.25 * (L - w)) < 1e-12


def test_decoupled_ring_smaller_than_gpu_set(solve):
    # transfers hide behind 2 layers (d = 2) but the CPU needs >= 7 GPU-optimised layers (eq. 3)
    L = 10
    prof = homog(L, 1.0, 1.5, 1.0, t_stage=[0.1] * L, t_opt_cpu=[10.0] * L, t_opt_gpu=[0.1] * L)
    coupled = solve(**prof, cpu_hard=True)
    dec = solve(**prof, cpu_hard=True, decouple=True)
    gmin = math.ceil((10 * L - 4 * L) / 10.1)
    assert coupled["window"] == gmin and coupled["ring_slots"] == gmin + 1
    assert dec["window"] == gmin and dec["ring_slots"] == 3
    # memory: the decoupled choice fits where the coupled one would not
    prof_mem = dict(prof, slot_bytes=[10] * L, gstate_bytes=[1] * L, s_avail=3 * 10 + gmin * 1)
    assert solve(**prof_mem, cpu_hard=True, decouple=True)["window"] == gmin
    assert solve(**prof_mem, cpu_hard=True)["window"] < gmin


def test_fp_serial_homogeneous_closed_form(solve):
    """R23 by hand: t_fp = a < t_c2g = c, no CPU constraint, decoupled (g = d).  The host fetches
    (layers d..L-1) are link-bound from the step start: fetch j lands at (j - d + 1) c and is due at
    S(j) = j a; the last layer binds: (L - d) c <= (L - 1) a  <=>  d >= L - (L - 1) a / c.  Together with
    (1b) d a >= c and (2b) 3 d a >= c: d* = max(ceil(c / a), ceil(L - (L - 1) a / c))."""
    for L, a, c in [(20, 1.0, 1.5), (40, 2.0, 3.0), (30, 1.0, 1.1), (16, 1.0, 4.0)]:
        prof = homog(L, a, c, 0.0, t_stage=[0.0] * L)
        d_star = max(math.ceil(c / a - 1e-12), math.ceil(L - (L - 1) * a / c - 1e-12))
        got = solve(**prof, decouple=True, fp_serial=True)
        assert got["ring_slots"] == d_star + 1 and got["window"] == d_star, (L, a, c, got, d_star)
        # without the serial form the paper's (1b) alone accepts a much shorter ring
        assert solve(**prof, decouple=True)["ring_slots"] == math.ceil(c / a - 1e-12) + 1


def test_fill_gpu_takes_the_memory_left_by_the_ring(solve):
    L = 12
    prof = homog(L, 1.0, 0.5, 0.5, t_stage=[0.0] * L, slot_bytes=[10] * L, gstate_bytes=[3] * L, s_avail=20 + 3 * 7)
    small = solve(**prof, decouple=True)
    full = solve(**prof, decouple=True, fill_gpu=True)
    assert small["ring_slots"] == full["ring_slots"] == 2       # d = 1: (1b) t_fp >= t_c2g
    assert small["window"] == 1 and full["window"] == 7         # 2 slots x 10 + 7 x 3 = 41 bytes


def test_link_bound_pool_sized_ring(solve):
    """R27 by hand: homogeneous, t_fp = 1 < t_c2g = 4 (every ring fails the serial form of (1b): the FP is
    link-bound), t_bp = 3, t_opt_cpu = 30 (BP outruns the CPU: backlog 1 - 3/30 = 0.9 per host layer),
    1 landing buffer, slots of 1 byte and GPU states of 10 bytes in S_avail = 300, decoupled + fill_gpu.
    g_for(d) = floor((300 - (d + 1)) / 10); the pool of d + 1 grad halves must hold
    B = ceil(0.9 (L - g)) - 1; the per-window (1b) needs d >= 4."""
    L, D = 40, 1
    prof = homog(L, 1.0, 4.0, 0.0, t_stage=[0.0] * L, t_opt_cpu=[30.0] * L, slot_bytes=[1] * L,
                 gstate_bytes=[10] * L, s_avail=300)
    want = None
    for d in range(L):
        g = min(L, (300 - (d + 1)) // 10)
        if d >= 4 and d + 1 >= math.ceil(0.9 * (L - g) - 1e-9) - D:
            want = (d, g)
            break
    assert want == (8, 29)
    r = solve(**prof, decouple=True, fp_serial=True, fill_gpu=True, landing_buffers=D)
    assert (r["ring_slots"] - 1, r["window"], r["reason"]) == (want[0], want[1], 3), r
    # without the landing-buffer count the solver keeps the memory fallback (coupled)
    r0 = solve(**prof, decouple=True, fp_serial=True, fill_gpu=True)
    assert r0["reason"] == 2 and r0["ring_slots"] == r0["window"] + 1


@pytest.mark.parametrize("seed", range(60))
def test_random_heterogeneous_matches_bruteforce(seed):
    rng = np.random.default_rng(seed)
    L = int(rng.integers(1, 30))
    prof = dict(t_fp=rng.uniform(0.1, 3, L), t_bp=rng.uniform(0.3, 9, L), t_c2g=rng.uniform(0, 6, L),
                t_g2c=rng.uniform(0, 8, L), t_stage=rng.uniform(0, 0.5, L), t_opt_gpu=rng.uniform(0, 1, L),
                t_opt_cpu=rng.uniform(0, 20, L), t_async=float(rng.uniform(0, 0.1)),
                slot_bytes=rng.integers(1, 100, L), gstate_bytes=rng.integers(1, 60, L),
                fixed_bytes=int(rng.integers(0, 50)), s_avail=int(rng.integers(100, 3000)),
                duplex=bool(rng.integers(0, 2)), cpu_hard=bool(rng.integers(0, 2)),
                cpu_util_max=float(rng.choice([1.0, 0.85, 0.5])), decouple=bool(rng.integers(0, 2)),
                fp_serial=bool(rng.integers(0, 2)), fill_gpu=bool(rng.integers(0, 2)),
                landing_buffers=int(rng.integers(0, 6)))
    want = AO.solve(**{k: (list(v) if isinstance(v, np.ndarray) else v) for k, v in prof.items()})
    if want is None:
        with pytest.raises(sh.ShError):
            sh.solve_window(**prof)
        return
    got = sh.solve_window(**prof)
    for k in ("window", "reason", "w_max_memory", "ring_slots"):
        assert got[k] == want[k], (k, got, want)
    for k in ("eq3_min_slack_ms", "eq4_lhs_ms", "eq4_rhs_ms"):
        assert abs(got[k] - want[k]) <= 1e-9 * max(1.0, abs(want[k])), (k, got, want)


@pytest.mark.parametrize("seed", range(40))
def test_random_link_bound_profiles_match_bruteforce(seed):
    """Profiles where the FP is link-bound (t_c2g >> t_fp) and the GPU set fills the memory, so the R27
    tier decides: the C++ solver agrees with the brute-force oracle."""
    rng = np.random.default_rng(1000 + seed)
    L = int(rng.integers(8, 40))
    prof = dict(t_fp=rng.uniform(0.5, 1.5, L), t_bp=rng.uniform(1.5, 4.5, L), t_c2g=rng.uniform(2.0, 6.0, L),
                t_g2c=rng.uniform(0, 4, L), t_stage=rng.uniform(0, 0.2, L), t_opt_cpu=rng.uniform(3, 30, L),
                slot_bytes=[int(rng.integers(1, 4))] * L, gstate_bytes=rng.integers(5, 15, L),
                s_avail=int(rng.integers(60, 400)), decouple=True, fp_serial=True, fill_gpu=True,
                landing_buffers=int(rng.integers(1, 8)))
    want = AO.solve(**{k: (list(v) if isinstance(v, np.ndarray) else v) for k, v in prof.items()})
    if want is None:
        with pytest.raises(sh.ShError):
            sh.solve_window(**prof)
        return
    got = sh.solve_window(**prof)
    for k in ("window", "reason", "w_max_memory", "ring_slots"):
        assert got[k] == want[k], (k, got, want)
