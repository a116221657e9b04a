"""Writes tests/golden/beaver_*.json -- worked examples of PAPER.md Sec. 2.2 (Eqs. 1-6).

The paper prints no numeric example, so these fixtures are produced by this
committed script from oracle/ only: inputs, shares and triplets come from the oracle's ChaCha20
PRG streams (R1, R4); every expected value (E_i, E, F_i, F, C_i for the BJ form and
Eq. 6, the reconstruction A.B, the truncated shares) is computed with Python big integers in
oracle/bruteforce.py, independently of the C oracle's uint64 arithmetic.

    python tests/golden/make_golden.py
"""
import json
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(os.path.dirname(HERE)))

from oracle import bruteforce as bf  # noqa: E402
from oracle import core  # noqa: E402

SEED = 0x50534D4C


def ints(a):
    return [[int(v) for v in row] for row in a]


def make(l, M, K, N, trunc):
    cid = (M << 16) | (K << 8) | N
    A = core.prg(l, SEED, core.tag("gA"), cid, M * K).reshape(M, K)
    B = core.prg(l, SEED, core.tag("gB"), cid, K * N).reshape(K, N)
    A0, A1 = core.share(A, SEED + 1, cid * 2, l)
    B0, B1 = core.share(B, SEED + 1, cid * 2 + 1, l)
    U0, U1, V0, V1, Z0, Z1 = core.triplet_gen(SEED + 2, cid, M, K, N, l)
    E0, E1 = bf.add_mod(A0, U0, l, -1), bf.add_mod(A1, U1, l, -1)
    F0, F1 = bf.add_mod(B0, V0, l, -1), bf.add_mod(B1, V1, l, -1)
    E, F = bf.add_mod(E0, E1, l), bf.add_mod(F0, F1, l)
    C = [bf.beaver_shares_bj(E, F, (U0, U1)[i], (V0, V1)[i], (Z0, Z1)[i], i, l) for i in range(2)]
    P = [bf.beaver_shares_paper(E, F, (A0, A1)[i], (B0, B1)[i], (Z0, Z1)[i], i, l)
         for i in range(2)]
    T = [[[bf.truncate_share(v, i, trunc, l) for v in row] for row in C[i]] for i in range(2)]
    return dict(
        citation="PAPER.md L65-L78 (Sec. 2.2, Eqs. 1-6); BJ canonical form C_i = i.E.F + E.V_i + "
                 "U_i.F + Z_i; truncation = SecureML local (DESIGN.md R7)",
        l=l, M=M, K=K, N=N, trunc=trunc,
        A=ints(A), B=ints(B), A0=ints(A0), A1=ints(A1), B0=ints(B0), B1=ints(B1),
        U0=ints(U0), U1=ints(U1), V0=ints(V0), V1=ints(V1), Z0=ints(Z0), Z1=ints(Z1),
        E0=E0, E1=E1, E=E, F0=F0, F1=F1, F=F, C0=C[0], C1=C[1], P0=P[0], P1=P[1],
        T0=T[0], T1=T[1], AB=bf.matmul_mod(ints(A), ints(B), l))


if __name__ == "__main__":
    for l in (8, 16, 32, 64):
        for (M, K, N) in ((4, 4, 4), (3, 5, 2)):
            d = make(l, M, K, N, trunc=3 if l <= 16 else 13)
            with open(os.path.join(HERE, f"beaver_l{l}_{M}x{K}x{N}.json"), "w") as f:
                json.dump(d, f)
    print("ok")
