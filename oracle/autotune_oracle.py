"""Brute-force transcription of the paper's window model -- TEST INFRASTRUCTURE ONLY.

PAPER.md:132-195 (§III-D): P1 (eq. 1a-1d), P2 (eq. 2a-2d), the window rule,
eq. 3 and eq. 4.  Plain nested loops over layers for every candidate m, no prefix sums and no
code shared with the C++ solver (paper_conf_sc_sunwqyhxw22_b200/csrc/autotune.cpp).  Readings
(R4-R8, R19) are the same, stated here again next to the formulas:

  m = w = prefetch distance; ring w+1 slots;  memory (1c)/(2c):
      fixed + (w+1) * max_i slot_bytes_i + sum_{i<w} gstate_bytes_i <= S_avail
  (1b) for every layer j entering the FP window (j = w..L-1):
      sum_{i=j-w}^{j-1} t_fp[i] >= t_c2g[j]
  (2b) for every layer j entering the BP window (j = L-w-2..0):
      sum_{i=j+1}^{j+w} t_bp[i] >= max(t_g2c[j+w+1], t_stage[j] if j < w else t_c2g[j])
  (1d) sum over the same FP windows: sum t_fp >= sum t_c2g + sum t_g2c   (max() if duplex)
  (2d) sum over the same BP windows: sum t_bp >= sum t_c2g + sum t_g2c   (max() if duplex)
  rule: min{w < L : mem & hard & soft}, else min{w <= L : mem & hard}, else max{w : mem}
  decouple (R22): prefetch distance d (ring d+1) and GPU-optimised set g = max(d, g_min) separately;
      (1b)/(2b) fetch cost of a GPU-optimised layer is t_stage, and it has no offload (g2c = 0)
  cpu_hard (optional): sum_{k>=w} t_opt_cpu[k] <= rho (sum_i (t_fp[i] + t_bp[i]) + sum_{i<w} t_opt_gpu[i])
  eq. 3 slack: min_{k in [w, L)} [ sum_{i<=k}(t_fp[i]+t_bp[i]) + sum_{i<w} t_opt_gpu[i] - t_opt_cpu[k] ]
  eq. 4: 5 L t_async  vs  sum_{i=w}^{L-1} t_opt_gpu[i]
  fp_serial (R23, decoupled or not): the FP fetches of host layers j = g..L-1 queue on one link:
      S(p) = sum_{i<p} t_fp[i] (compute start of FP position p with no stall)
      F(j) = max(F(j-1), S(max(0, j-d))) + t_c2g[j]   (slot of position j-d-1 free, link free)
      hard: F(j) <= S(j) for every host layer j
  fill_gpu (decoupled): g = the largest g >= max(d, g_min) that fits next to the ring, not the smallest
  link-bound fallback (R27, decoupled + fill_gpu + landing_buffers > 0, no (d, g) meets the hard
      constraints): the smallest d whose ring d+1 holds the backward backlog
      B(g) = ceil(sum_{k>=g} max(0, 1 - t_bp[k] / t_opt_cpu[k])) - landing_buffers, g = the largest GPU set
      the memory leaves next to the ring (no CPU constraint: the CPU is then the bottleneck anyway), with
      the per-window (1b) / (2b) met -> reason 3
"""
from __future__ import annotations

import math


def _z(a, n):
    return [0.0] * n if a is None else [float(x) for x in a]


def solve(t_fp, t_bp, t_c2g, t_g2c, t_stage=None, t_opt_gpu=None, t_opt_cpu=None, t_async=0.0,
          slot_bytes=None, gstate_bytes=None, fixed_bytes=0, s_avail=2 ** 62, duplex=False, cpu_hard=False,
          cpu_util_max=1.0, decouple=False, fp_serial=False, fill_gpu=False, landing_buffers=0):
    """d = prefetch distance (ring d+1 slots), g = GPU-optimised layers [0, g); coupled d = g = m
    (the paper), decoupled g = max(d, smallest g meeting the CPU constraint) (R22)."""
    L = len(t_fp)
    fp, bp, c2g, g2c = _z(t_fp, L), _z(t_bp, L), _z(t_c2g, L), _z(t_g2c, L)
    st, og, oc = _z(t_stage, L), _z(t_opt_gpu, L), _z(t_opt_cpu, L)
    sb = [0] * L if slot_bytes is None else list(slot_bytes)
    gb = [0] * L if gstate_bytes is None else list(gstate_bytes)

    def mem(d, g):
        need = fixed_bytes + (d + 1) * max(sb)
        for i in range(g):
            need += gb[i]
        return need <= s_avail

    def fetch(j, g):
        return st[j] if j < g else c2g[j]

    def fp_hard(d, g):
        for j in range(d, L):
            s = 0.0
            for i in range(j - d, j):
                s += fp[i]
            if s < fetch(j, g):
                return False
        return True

    def bp_hard(d, g):
        for j in range(L - d - 2, -1, -1):
            s = 0.0
            for i in range(j + 1, j + d + 1):
                s += bp[i]
            off = g2c[j + d + 1] if j + d + 1 >= g else 0.0   # GPU-optimised layers are not offloaded
            if s < max(off, fetch(j, g)):
                return False
        return True

    def window_ok(times, lo, hi):
        comp = sum(times[i] for i in range(lo, hi))
        a = sum(c2g[i] for i in range(lo, hi))
        b = sum(g2c[i] for i in range(lo, hi))
        return comp >= (max(a, b) if duplex else a + b)

    def soft(d):
        for j in range(d, L):
            if not window_ok(fp, j - d, j):
                return False
        for j in range(L - d - 2, -1, -1):
            if not window_ok(bp, j + 1, j + d + 1):
                return False
        return True

    def cpu_ok(g):
        if not cpu_hard:
            return True
        rho = cpu_util_max if 0.0 < cpu_util_max < 1.0 else 1.0
        return sum(oc[k] for k in range(g, L)) <= rho * (sum(fp) + sum(bp) + sum(og[:g]))

    def serial_ok(d, g):
        if not fp_serial:
            return True
        F = None
        for j in range(g, L):
            q = max(0, j - d)
            slot_free = 0.0
            for i in range(q):
                slot_free += fp[i]
            start = slot_free if F is None else max(F, slot_free)
            F = start + c2g[j]
            s_j = 0.0
            for i in range(j):
                s_j += fp[i]
            if F > s_j:
                return False
        return True

    def hard(d, g):
        return fp_hard(d, g) and bp_hard(d, g) and cpu_ok(g) and serial_ok(d, g)

    mems = [w for w in range(L + 1) if mem(w, w)]
    if not mems:
        return None
    best = None
    reason = 2
    if not decouple:
        for w in range(L):
            if mem(w, w) and hard(w, w) and soft(w):
                best, reason = (w, w), 0
                break
        if best is None:
            for w in range(L + 1):
                if mem(w, w) and hard(w, w):
                    best, reason = (w, w), 1
                    break
    else:
        gmin = 0
        while gmin < L and not cpu_ok(gmin):
            gmin += 1

        def g_for(d):
            cands = [x for x in range(max(d, gmin), L + 1) if mem(d, x)]
            if not cands:
                return None
            return max(cands) if fill_gpu else (max(d, gmin) if mem(d, max(d, gmin)) else None)

        for d in range(L):
            g = g_for(d)
            if g is not None and hard(d, g) and soft(d):
                best, reason = (d, g), 0
                break
        if best is None:
            for d in range(L + 1):
                g = g_for(d)
                if g is not None and hard(d, g):
                    best, reason = (d, g), 1
                    break
        if best is None and fill_gpu and landing_buffers > 0:
            def backlog(g):
                b = 0.0
                for k in range(g, L):
                    if oc[k] > 0:
                        b += max(0.0, 1.0 - bp[k] / oc[k])
                return math.ceil(b - 1e-9) - landing_buffers

            for d in range(L + 1):
                fits = [x for x in range(d, L + 1) if mem(d, x)]
                g = max(fits) if fits else None
                if g is not None and d + 1 >= backlog(g) and fp_hard(d, g) and bp_hard(d, g):
                    best, reason = (d, g), 3
                    break
    if best is None:
        best = (max(mems), max(mems))
    d, g = best
    slack = None
    for k in range(g, L):
        rhs = sum(fp[i] + bp[i] for i in range(k + 1)) + sum(og[i] for i in range(g))
        v = rhs - oc[k]
        slack = v if slack is None else min(slack, v)
    cpu_total = 0.0
    for k in range(g, L):
        cpu_total += oc[k]
    gpu_step = sum(fp[i] + bp[i] for i in range(L)) + sum(og[i] for i in range(g))
    return {"window": g, "ring_slots": d + 1, "reason": reason, "w_max_memory": max(mems),
            "cpu_total_ms": cpu_total, "gpu_step_ms": gpu_step,
            "eq3_min_slack_ms": 0.0 if slack is None else slack,
            "eq4_lhs_ms": 5.0 * L * t_async, "eq4_rhs_ms": sum(og[i] for i in range(g, L))}
