"""Model of the P-rank critical path of the 1D block-cyclic distributed factorisation at C4
(DESIGN.md §5): per iteration k the step takes max(U_k / P, panel_{k+1}) — every rank applies its
share of update k while the owner of column k+1 runs its panel chain (look-ahead depth 1).

Inputs are the single-GPU measurements quoted in DESIGN.md §5/§7 (C4, n = 32768, nb = 512):
363 ms of update per factorisation (bulk-copy producer; the LDGSTS producer is `ldg` times
slower), the TRSM 13.7 ms in total, checks 0.25 ms per panel, write-back at 6 TB/s, broadcast at
700 GB/s. Usage: python tools/p_model.py
"""
import sys

n, nb = 32768, 512
N = n // nb
U_TOTAL, TRSM_TOTAL, CHECKS = 363.0, 13.7, 0.25     # ms
WB_BW, BC_BW = 6.0e9, 0.7e9                          # bytes per ms


def step_ms(P, diag_ms, ldg=1.0):
    ms = [N - k - 1 for k in range(N)]
    s2, s1 = sum(m * m for m in ms), sum(ms)
    t, bound = 0.0, 0

    def panel(k):
        m = ms[k]
        w = (m * nb + 2 * m + 2) * nb * 8
        return diag_ms + TRSM_TOTAL * m / s1 + CHECKS + w / WB_BW + (w / BC_BW if P > 1 else 0.0)

    t += panel(0)
    for k in range(N):
        u = ldg * U_TOTAL * ms[k] ** 2 / s2 / P
        p = panel(k + 1) if k + 1 < N else 0.0
        if p > u:
            bound += 1
        t += max(u, p)
    return t, bound


def main():
    flops = n ** 3 / 3
    rows = []
    base1 = step_ms(1, 0.89)[0]
    print("| P | recursive diagonal block (0.89 ms), bulk-copy update | panel-bound | "
          "task-graph diagonal block (0.25 ms), LDGSTS update (x1.09) | panel-bound |")
    print("|---|---|---|---|---|")
    for P in (1, 2, 4, 8):
        a, ba = step_ms(P, 0.89)
        b, bb = step_ms(P, 0.25, 1.09)
        ea = base1 / (P * a)
        eb = base1 / (P * b)
        rows.append((P, a, b))
        print(f"| {P} | {a:.0f} ms ({flops / a / 1e9:.1f} TFLOP/s, {100 * ea:.0f} % of linear) | {ba} / {N} | "
              f"{b:.0f} ms ({flops / b / 1e9:.1f} TFLOP/s, {100 * eb:.0f} %) | {bb} / {N} |")
    return rows


if __name__ == "__main__":
    sys.exit(0 if main() else 1)
