"""Writes tests/golden/c4_nchk3_events.txt: the ORACLE's event list for C4 (n=32768, nb=512) with
three checksum rows (NEXT-4, reading B10) under the C3-style mixed injections plus a second error
next to every tenth one (bit <= 58), the recipe bench.py's next4_three_checksums run uses. Calls
only oracle/ and synthetic/ (about 8 minutes on 8 cores); the GPU test compares against it.
usage: python tests/golden/make_c4_nchk3_events.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import synthetic as syn  # noqa: E402


def recipe(n, nb):
    return syn.next4_injections(n, nb)


if __name__ == "__main__":
    n, nb = 32768, 512
    r = oracle.potrf(syn.spd_matrix(n), nb, inj=syn.inj_array(recipe(n, nb)), nchk=3)
    out = os.path.join(os.path.dirname(os.path.abspath(__file__)), "c4_nchk3_events.txt")
    with open(out, "w") as f:
        f.write(f"# oracle status {r.status}; (k, check, tile_j, tile_i, col, row, kind, rank) per event\n")
        for e in r.event_tuples():
            f.write(" ".join(str(v) for v in e) + "\n")
    print(out, r.status, len(r.events))
