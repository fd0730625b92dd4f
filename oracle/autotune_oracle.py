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
  cpu_hard (optional): sum_{k>=w} t_opt_cpu[k] <= rho (sum_i (t_fp[i] + t_bp[i]) + sum_{i<w} t_opt_gpu[i])
  eq. 3 slack: min_{k in [w, L)} [ sum_{i<=k}(t_fp[i]+t_bp[i]) + sum_{i<w} t_opt_gpu[i] - t_opt_cpu[k] ]
  eq. 4: 5 L t_async  vs  sum_{i=w}^{L-1} t_opt_gpu[i]
"""
from __future__ import annotations


def _z(a, n):
    return [0.0] * n if a is None else [float(x) for x in a]


def solve(t_fp, t_bp, t_c2g, t_g2c, t_stage=None, t_opt_gpu=None, t_opt_cpu=None, t_async=0.0,
          slot_bytes=None, gstate_bytes=None, fixed_bytes=0, s_avail=2 ** 62, duplex=False, cpu_hard=False,
          cpu_util_max=1.0):
    L = len(t_fp)
    fp, bp, c2g, g2c = _z(t_fp, L), _z(t_bp, L), _z(t_c2g, L), _z(t_g2c, L)
    st, og, oc = _z(t_stage, L), _z(t_opt_gpu, L), _z(t_opt_cpu, L)
    sb = [0] * L if slot_bytes is None else list(slot_bytes)
    gb = [0] * L if gstate_bytes is None else list(gstate_bytes)

    def mem(w):
        need = fixed_bytes + (w + 1) * max(sb)
        for i in range(w):
            need += gb[i]
        return need <= s_avail

    def fp_hard(w):
        for j in range(w, L):
            s = 0.0
            for i in range(j - w, j):
                s += fp[i]
            if s < c2g[j]:
                return False
        return True

    def bp_hard(w):
        for j in range(L - w - 2, -1, -1):
            s = 0.0
            for i in range(j + 1, j + w + 1):
                s += bp[i]
            fetch = st[j] if j < w else c2g[j]
            if s < max(g2c[j + w + 1], fetch):
                return False
        return True

    def window_ok(times, lo, hi):
        comp = sum(times[i] for i in range(lo, hi))
        a = sum(c2g[i] for i in range(lo, hi))
        b = sum(g2c[i] for i in range(lo, hi))
        return comp >= (max(a, b) if duplex else a + b)

    def soft(w):
        for j in range(w, L):
            if not window_ok(fp, j - w, j):
                return False
        for j in range(L - w - 2, -1, -1):
            if not window_ok(bp, j + 1, j + w + 1):
                return False
        return True

    def cpu_ok(w):
        if not cpu_hard:
            return True
        rho = cpu_util_max if 0.0 < cpu_util_max < 1.0 else 1.0
        return sum(oc[k] for k in range(w, L)) <= rho * (sum(fp) + sum(bp) + sum(og[:w]))

    def hard(w):
        return fp_hard(w) and bp_hard(w) and cpu_ok(w)

    mems = [w for w in range(L + 1) if mem(w)]
    if not mems:
        return None
    best, reason = None, 2
    for w in range(L):
        if mem(w) and hard(w) and soft(w):
            best, reason = w, 0
            break
    if best is None:
        for w in range(L + 1):
            if mem(w) and hard(w):
                best, reason = w, 1
                break
    if best is None:
        best = max(mems)
    slack = None
    for k in range(best, L):
        rhs = sum(fp[i] + bp[i] for i in range(k + 1)) + sum(og[i] for i in range(best))
        v = rhs - oc[k]
        slack = v if slack is None else min(slack, v)
    return {"window": best, "reason": reason, "w_max_memory": max(mems),
            "eq3_min_slack_ms": 0.0 if slack is None else slack,
            "eq4_lhs_ms": 5.0 * L * t_async, "eq4_rhs_ms": sum(og[i] for i in range(best, L))}
