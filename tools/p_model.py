"""Model of the P-rank critical path of the distributed factorisation at C4: per
iteration k the step takes max(U_k / P, panel_{k+1}) — every rank applies its share of update k
while the owners of column k+1 run the panel chain (look-ahead depth 1).

Inputs are single-GPU measurements at C4 (n = 32768, nb = 512; profiles/r02/bench_r02_final.jsonl):
366 ms of update per factorisation, the diagonal block 20.2 ms in total (task graph, 0.32 ms per
block), the TRSM 14.9 ms in total, checks 0.25 ms per panel, write-back at 6 TB/s; links at 700
GB/s per direction (NVLink 5 usable).
  1D: the owner of column k solves the whole panel and broadcasts it (NCCL: ~ w / link bandwidth).
  2D (Pr x Pc grid, peer-memory push): the diagonal block's owner pushes inv(L_kk) (nb^2 doubles) to
      its process column, each of the Pr column ranks solves 1/Pr of the panel and pushes its rows to
      the P - 1 other ranks (egress w (P - 1) / Pr per contributor, ingress w per receiver).
Usage: python tools/p_model.py
"""
import sys

n, nb = 32768, 512
N = n // nb
U_TOTAL, DIAG_TOTAL, TRSM_TOTAL, CHECKS = 366.4, 20.2, 14.9, 0.25   # ms
WB_BW, LINK = 6.0e9, 0.7e9                                          # bytes per ms


def step_ms(P, Pr=1):
    ms = [N - k - 1 for k in range(N)]
    s2, s1 = sum(m * m for m in ms), sum(ms)
    diag = DIAG_TOTAL / N
    t, bound = 0.0, 0

    def panel(k):
        m = ms[k]
        w = (m * nb + 2 * m + 2) * nb * 8
        if P == 1:
            return diag + TRSM_TOTAL * m / s1 + CHECKS + w / WB_BW
        if Pr == 1:   # owner solves everything, broadcast
            return diag + TRSM_TOTAL * m / s1 + CHECKS + w / WB_BW + w / LINK
        li = nb * nb * 8 / LINK
        push = max(w * (P - 1) / Pr / LINK, w / LINK)
        return diag + li + TRSM_TOTAL * m / s1 / Pr + CHECKS + w / Pr / WB_BW + push

    t += panel(0)
    for k in range(N):
        u = U_TOTAL * ms[k] ** 2 / s2 / P
        p = panel(k + 1) if k + 1 < N else 0.0
        if p > u:
            bound += 1
        t += max(u, p)
    return t, bound


def main():
    flops = n ** 3 / 3
    base1 = step_ms(1)[0]
    print("| P | grid | modelled step | TFLOP/s | of linear | panel-bound iterations |")
    print("|---|---|---|---|---|---|")
    rows = []
    for P, Pr in ((1, 1), (2, 1), (2, 2), (4, 1), (4, 2), (8, 1), (8, 2), (8, 4)):
        t, b = step_ms(P, Pr)
        grid = "1" if P == 1 else (f"1D x{P}" if Pr == 1 else f"2D {Pr}x{P // Pr}")
        rows.append((P, Pr, t))
        print(f"| {P} | {grid} | {t:.0f} ms | {flops / t / 1e9:.1f} | {100 * base1 / (P * t):.0f} % | {b} / {N} |")
    return rows


if __name__ == "__main__":
    sys.exit(0 if main() else 1)
