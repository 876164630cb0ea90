"""Ground truth for single injections: which check must see an error injected at a hook, and
where it must locate it. Derived from the verification schedule of the paper's Enhanced
Online-ABFT (§III: verify each block before it is referenced; Table I,
PAPER.md:257-265) as laid out in SURVEY.md §8c step 2 (V1..V6), not from any implementation.

  hook REST(k)       element in tile (I,J):  J <  k -> V6 (finished L, next reader is the caller)
                                             J == k -> V1 (I == k) / V2 (I > k) at k
                                             J >  k -> V5 at k (the tile enters the update additively)
  hook POTRF_OUT(k)  tile (k,k)              -> V3 at k
  hook TRSM_OUT(k)   tile (I>k, k)           -> V4 at k
  hook UPDATE_OUT(k) tile (I>=J>k)           -> V5 at k
  hook REST(N)                               -> V6 at N
Location: d1 = Delta, d2 = (r+1) Delta -> data row r; an error in checksum
row 1 / row 2 shows as d1 alone / d2 alone (CHK1 / CHK2, reading A10).
"""

V = {"V1": 1, "V2": 2, "V3": 3, "V4": 4, "V5": 5, "V6": 6, "V4R": 7, "V7": 8}
KIND = {"DATA": 1, "NONFINITE": 2, "CHK1": 3, "CHK2": 4, "UNCORRECTABLE": 5, "CHK3": 6}
HOOKS = {"REST": 0, "POTRF_OUT": 1, "TRSM_OUT": 2, "UPDATE_OUT": 3, "RECV": 4}


def predict_left(spec, n, nb, K=1):
    """Left-looking order (MAGMA Alg. 1) with Table I's verification:
    iteration j verifies A[j,j] and B = A[j+1:,j] (V1/V2) and the L blocks it reads, C = L[j,0:j] and
    D = L[j+1:,0:j] (V7, D every K iterations), the updated column (V5), L[j,j] (V3); V6 at the end.
      REST(j) in tile (I,J): J == j -> V1/V2 at j; J > j -> V1/V2 at J (untouched until then);
                             J < j -> V7 at the first j' >= j reading it (I >= j', D gated), else V6
      UPDATE_OUT(j) -> V5 at j;  POTRF_OUT(j) -> V3 at j;  TRSM_OUT(j) -> V7 at the next read"""
    N = n // nb
    k = spec["k"]
    hook = spec["hook"] if isinstance(spec["hook"], str) else {v: kk for kk, v in HOOKS.items()}[spec["hook"]]
    r, c = spec["row"], spec["col"]
    I, J = r // nb, c // nb
    row, col, kind = r - I * nb, c - J * nb, KIND["DATA"]

    def first_read(j0):
        for jj in range(j0, N):
            if jj > J and I >= jj and (I == jj or jj % K == 0):
                return (jj, V["V7"])
        return (N, V["V6"])

    if hook == "REST":
        if k >= N:
            ck, v = N, V["V6"]
        elif J >= k:
            ck, v = J, V["V1"] if I == J else V["V2"]
        else:
            ck, v = first_read(k)
    elif hook == "UPDATE_OUT":
        ck, v = k, V["V5"]
    elif hook == "POTRF_OUT":
        ck, v = k, V["V3"]
    elif hook == "TRSM_OUT":
        ck, v = first_read(k + 1)
    else:
        raise ValueError(hook)
    return (ck, v, J, I, col, row, kind, 0)


def predict(spec, n, nb, K=1, nchk=2):
    """Return the expected event tuple (k, V, J, I, col, row, kind, rank) for one injection.
    nchk: checksum rows per block (checksum-row targets are rows nchk*I + t; t = 2 -> CHK3)."""
    N = n // nb
    k = spec["k"]
    hook = spec["hook"] if isinstance(spec["hook"], str) else {v: kk for kk, v in HOOKS.items()}[spec["hook"]]
    tgt = spec.get("target", "DATA")
    if tgt == "DATA":
        r, c = spec["row"], spec["col"]
        I, J = r // nb, c // nb
        row, col = r - I * nb, c - J * nb
        kind = KIND["DATA"]
    else:
        cr, c = spec["row"], spec["col"]
        I, J = cr // nchk, c // nb
        col = c - J * nb
        row = (-1, -2, -4)[cr % nchk]
        kind = (KIND["CHK1"], KIND["CHK2"], KIND["CHK3"])[cr % nchk]
    if hook == "REST":
        if k >= N or J < k:
            chk_k, v = N, V["V6"]
        elif J == k:
            chk_k, v = k, V["V1"] if I == k else V["V2"]
        else:
            # Opt. 3: V5 runs only at gated iterations k' (k'+1 = 0 mod K, or
            # the last update k' = N-2); if none falls in [k, J-1], V1/V2 at J reads it first.
            gated = [kk for kk in range(k, J) if (kk + 1) % K == 0 or kk == N - 2]
            if gated:
                chk_k, v = gated[0], V["V5"]
            else:
                chk_k, v = J, V["V1"] if I == J else V["V2"]
    elif hook == "POTRF_OUT":
        chk_k, v = k, V["V3"]
    elif hook == "TRSM_OUT":
        chk_k, v = k, V["V4"]
    elif hook == "UPDATE_OUT":
        gated = [kk for kk in range(k, J) if (kk + 1) % K == 0 or kk == N - 2]
        chk_k, v = (gated[0], V["V5"]) if gated else (J, V["V1"] if I == J else V["V2"])
    elif hook == "RECV":
        chk_k, v = k, V["V4R"]
    else:
        raise ValueError(hook)
    return (chk_k, v, J, I, col, row, kind, spec.get("rank", 0) if hook == "RECV" else 0)
