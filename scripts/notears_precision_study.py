"""NEXT-1: would the large-component penalty survive tensor-core
precision?  The library forms e^Abar - I for components above 64 classes on
CUDA-core fp64 GEMMs (kernels_notears.cu: scale by 2^-s, Horner expm1 of
degree 16, then s squarings Y <- Y^2 + 2Y).  This study runs the same
algorithm with every matrix product emulated in
  fp32      : fp32 inputs, fp32 accumulation (what 3xTF32 approximates),
  3xTF32    : hi = tf32(x), lo = tf32(x - hi); hi*hi + hi*lo + lo*hi, fp32 acc.,
  1xTF32    : tf32 inputs, fp32 accumulation (one tcgen05 kind::tf32 MMA),
on the Abar of the large-component test graphs (random logits U(-2, 2),
penalty groups of 8 seeds), and compares h = tr(e^Abar - I) and the penalty
gradient entries e^Abar[j, i] with fp64 against the parity bar
1e-6 + 1e-4 |ref|.  CPU only (numpy / scipy).

    python scripts/notears_precision_study.py   -> profiles/r2/notears_precision.md
"""
import os
import sys

import numpy as np
from scipy.sparse import csr_matrix
from scipy.sparse.csgraph import connected_components

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from gen import make_config  # noqa: E402

DEG = 16


def tf32(x):
    x = np.asarray(x, np.float32)
    b = x.view(np.uint32).astype(np.uint64)
    b = ((b + 0x1000) & 0xFFFFE000).astype(np.uint32)  # round to 10 explicit mantissa bits
    return b.view(np.float32)


def mm(a, b, mode):
    if mode == "fp64":
        return a @ b
    if mode == "fp32":
        return (a.astype(np.float32) @ b.astype(np.float32)).astype(np.float64)
    a32, b32 = a.astype(np.float32), b.astype(np.float32)
    ah, bh = tf32(a32), tf32(b32)
    if mode == "1xtf32":
        return (ah @ bh).astype(np.float64)
    al, bl = tf32(a32 - ah), tf32(b32 - bh)
    return (ah @ bh + (ah @ bl + al @ bh)).astype(np.float64)


def expm1_chain(A, s, mode):
    n = A.shape[0]
    X = A * 2.0 ** -s
    if mode != "fp64":
        X = X.astype(np.float32).astype(np.float64)
    I = np.eye(n)
    T = I + X / DEG
    for m in range(DEG - 1, 1, -1):
        T = I + mm(X, T, mode) / m
        if mode != "fp64":
            T = T.astype(np.float32).astype(np.float64)
    Y = mm(X, T, mode)
    for _ in range(s):
        Y = mm(Y, Y, mode) + 2 * Y
        if mode != "fp64":
            Y = Y.astype(np.float32).astype(np.float64)
    return Y


def abar_of_largest(eg, cp, G):
    M, N = eg.num_classes, eg.num_nodes
    ec = eg.ec()
    src = ec[np.repeat(np.arange(N), np.diff(eg.child_ptr))]
    dst = np.asarray(eg.child_class)
    A = csr_matrix((np.ones(len(src)), (src, dst)), shape=(M, M))
    _, lab = connected_components(A, directed=True, connection="strong")
    big = np.bincount(lab).argmax()
    mem = np.where(lab == big)[0]
    loc = -np.ones(M, np.int64)
    loc[mem] = np.arange(len(mem))
    n = len(mem)
    Ab = np.zeros((n, n))
    for k in range(N):
        i = ec[k]
        if loc[i] < 0:
            continue
        for j in set(eg.child_class[eg.child_ptr[k]:eg.child_ptr[k + 1]].tolist()):
            if loc[j] >= 0:
                Ab[loc[i], loc[j]] += cp[k, :G].mean()
    # structural squaring count of the library: rows sum to <= max_k |ch_k cap S|
    mx = 1
    for k in range(N):
        if loc[ec[k]] >= 0:
            mx = max(mx, sum(1 for j in set(eg.child_class[eg.child_ptr[k]:eg.child_ptr[k + 1]].tolist())
                             if loc[j] >= 0))
    s = int(np.ceil(np.log2(mx))) + 1
    return Ab, s


def main():
    rows = []
    for p_back in (0.06, 0.1, 0.15):
        eg = make_config("C2", scc_max=10**9, p_back=p_back)
        rng = np.random.default_rng(11)
        th = rng.uniform(-2, 2, (eg.num_nodes, 8))
        ec = eg.ec()
        cp = np.exp(th - th.max())
        den = np.zeros((eg.num_classes, 8))
        np.add.at(den, ec, cp)
        cp = cp / den[ec]
        A, s = abar_of_largest(eg, cp, 8)
        ref = expm1_chain(A, s, "fp64")
        h_ref = np.trace(ref)
        E_ref = ref + np.eye(len(A))
        for mode in ("fp32", "3xtf32", "1xtf32"):
            Y = expm1_chain(A, s, mode)
            E = Y + np.eye(len(A))
            h_err = abs(np.trace(Y) - h_ref) / abs(h_ref)
            ratio = np.abs(E - E_ref) / (1e-6 + 1e-4 * np.abs(E_ref))
            rows.append((p_back, len(A), s, mode, h_err, float(ratio.max()), float(np.mean(ratio <= 1))))
            print(rows[-1], flush=True)
    os.makedirs(os.path.join(ROOT, "profiles", "r2"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", "r2", "notears_precision.md"), "w") as fh:
        fh.write("# Large-component penalty at tensor-core precision (NEXT-1 study)\n\n")
        fh.write("`python scripts/notears_precision_study.py` (CPU emulation; see its docstring).  "
                 "Largest component of the C2 large-SCC test graphs, random logits, 8-seed groups; "
                 "the library's algorithm (2^-s scaling, Horner expm1 degree 16, s squarings) with "
                 "each product in the given precision, against fp64.\n\n")
        fh.write("| p_back | classes | squarings s | products | rel. error of h | worst entry / bar | entries within bar |\n")
        fh.write("|---|---|---|---|---|---|---|\n")
        for r in rows:
            fh.write(f"| {r[0]} | {r[1]} | {r[2]} | {r[3]} | {r[4]:.2e} | {r[5]:.3g} | {r[6]:.4f} |\n")


if __name__ == "__main__":
    main()
